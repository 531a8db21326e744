"""End-to-end preemption timeline on one clock: the host-clock <->
%globaltimer offset is measured NTP-style by tools/clock_sync_probe (before
and after, to bound drift), then C2 flag preemptions (armed and memop signal)
are timed from the host call (CLOCK_REALTIME) through the first warp seeing
the signal and the last warp's saved context (device stamps, shifted onto the
host clock) to ctxb_preempt returning.  GPU; prints a markdown table."""
import json
import os
import subprocess
import sys
import time

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def offset():
    exe = os.path.join(HERE, "clock_sync_probe")
    if not os.path.exists(exe):   # git-ignored build product
        subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-o", exe, exe + ".cu"], check=True)
    out = subprocess.run([exe], capture_output=True, text=True, check=True)
    return json.loads(out.stdout.strip().splitlines()[-1])


def main():
    o1 = offset()
    cfg = configs.c2()
    a = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    c = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    res = {}
    for name, fl in (("armed", cb.ARMED_SIGNAL), ("memop", 0)):
        prog = cb.Program(configs.c2_ir(), poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, flags=cb.ALL | fl)
        ctx = torch.empty(prog.context_capacity(296), dtype=torch.uint8, device="cuda")
        rows = []
        for fr in np.random.default_rng(3).uniform(0.1, 0.9, 16):
            run = prog.launch(296, [a, b, c], [], ctx, s)
            t0 = time.perf_counter()
            while time.perf_counter() < t0 + fr * 5.3e-3:
                pass
            h0 = time.time_ns()
            run.preempt(ctrl, stats=False)
            h1 = time.time_ns()
            hd = run.headers()
            pre = hd[:, 2] == 1
            if pre.any():
                stp = run.stamps()[pre].astype(np.int64)
                rows.append((h0, int(stp[:, 0].min()), int(stp[:, 1].max()), h1))
                run.resume(s)
            run.wait()
            del run
        res[name] = rows
    o2 = offset()

    def off_at(h):   # linear in host time between the two probes
        f = (h - o1["host_ns"]) / max(1, o2["host_ns"] - o1["host_ns"])
        return o1["offset_ns"] + f * (o2["offset_ns"] - o1["offset_ns"])
    print(f"offset before / after: {o1} / {o2}")
    lines = ["| signal | host call -> first warp sees the signal | first seen -> last context saved | "
             "last saved -> ctxb_preempt returns | host call -> return |", "|---|---|---|---|---|"]
    for name, rows in res.items():
        r = np.array(rows, dtype=np.float64)
        off = np.array([off_at(x) for x in r[:, 0]])
        a_ = (r[:, 1] - off - r[:, 0]) / 1e3
        b_ = (r[:, 2] - r[:, 1]) / 1e3
        c_ = (r[:, 3] - (r[:, 2] - off)) / 1e3
        d_ = (r[:, 3] - r[:, 0]) / 1e3
        lines.append(f"| {name} | {np.median(a_):.1f} µs | {np.median(b_):.1f} µs | {np.median(c_):.1f} µs | "
                     f"{np.median(d_):.1f} µs |")
    unc = max(o1["min_rtt_ns"], o2["min_rtt_ns"]) / 2e3
    drift = abs(o1["offset_ns"] - o2["offset_ns"]) / 1e3
    print("\n".join(lines))
    span = (o2["host_ns"] - o1["host_ns"]) / 1e9
    print(f"(offset uncertainty +-{unc:.1f} µs from the probe's min round trip; offset moved {drift:.1f} µs over "
          f"{span:.1f} s between the probes, interpolated linearly)")


if __name__ == "__main__":
    main()
