"""End-to-end preemption timeline on one clock: the host-clock <->
%globaltimer offset is measured NTP-style by tools/clock_sync_probe (before
and after, to bound drift), then C2 flag preemptions (armed and memop signal,
the watcher with and without the drain notice) are timed from the host call
(CLOCK_REALTIME) through the watcher raising the flag, the first warp seeing
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
    for name, fl in (("armed", cb.ARMED_SIGNAL), ("memop", 0), ("watcher", cb.WATCHER),
                     ("watcher + notice", cb.WATCHER | cb.DRAIN_NOTICE)):
        prog = cb.Program(configs.c2_ir(), poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, flags=cb.ALL | fl)
        grid = prog.persistent_grid()
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        rows = []
        for fr in np.random.default_rng(3).uniform(0.1, 0.9, 16):
            run = prog.launch(grid, [a, b, c], [], ctx, s)
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
                w = run.watcher_stamp() if fl & cb.WATCHER else 0
                rows.append((h0, int(stp[:, 0].min()), int(stp[:, 1].max()), h1, w or int(stp[:, 0].min()),
                             int(stp[:, 0].max())))
                run.resume(s)
            run.wait()
            del run
        res[name] = rows
    o2 = offset()

    def off_at(h):   # linear in host time between the two probes
        f = (h - o1["host_ns"]) / max(1, o2["host_ns"] - o1["host_ns"])
        return o1["offset_ns"] + f * (o2["offset_ns"] - o1["offset_ns"])
    print(f"offset before / after: {o1} / {o2}")
    lines = ["| signal | host call -> flag raised (watcher) | -> first warp sees the signal | first seen -> last seen | "
             "first seen -> last context saved | last saved -> ctxb_preempt returns | host call -> return |",
             "|---|---|---|---|---|---|---|"]
    for name, rows in res.items():
        r = np.array(rows, dtype=np.float64)
        off = np.array([off_at(x) for x in r[:, 0]])
        w_ = (r[:, 4] - off - r[:, 0]) / 1e3
        a_ = (r[:, 1] - r[:, 4]) / 1e3
        s_ = (r[:, 5] - r[:, 1]) / 1e3
        b_ = (r[:, 2] - r[:, 1]) / 1e3
        c_ = (r[:, 3] - (r[:, 2] - off)) / 1e3
        d_ = (r[:, 3] - r[:, 0]) / 1e3
        wt = f"{np.median(w_):.1f} µs" if "watcher" in name else "—"
        lines.append(f"| {name} | {wt} | {np.median(a_ if 'watcher' in name else w_ + a_):.1f} µs | "
                     f"{np.median(s_):.1f} µs | {np.median(b_):.1f} µs | {np.median(c_):.1f} µs | {np.median(d_):.1f} µs |")
    unc = max(o1["min_rtt_ns"], o2["min_rtt_ns"]) / 2e3
    drift = abs(o1["offset_ns"] - o2["offset_ns"]) / 1e3
    print("\n".join(lines))
    span = (o2["host_ns"] - o1["host_ns"]) / 1e9
    print(f"(offset uncertainty +-{unc:.1f} µs from the probe's min round trip; offset moved {drift:.1f} µs over "
          f"{span:.1f} s between the probes, interpolated linearly)")


if __name__ == "__main__":
    main()
