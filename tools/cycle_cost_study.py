"""What does one preempt -> resume cycle cost the preempted kernel?  For C2,
C3 and C4a on the library defaults (and FULL_HW): uninterrupted kernel time
T0 (median), then flag preemptions at random times, each followed by an L2
eviction and the resume; device overhead = (preempted launch's kernel time
+ resume launch's kernel time) - T0, and the host gap between the drain and
the resume kernel's start.  Usage: python tools/cycle_cost_study.py [trials]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def setups():
    c2 = configs.c2()
    A, B = (torch.from_numpy(c2["buffers"][n].view(np.int32)).cuda() for n in ("A", "B"))
    C = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    yield "c2", c2["ir"], 2, [A, B, C]
    if os.environ.get("ONLY_C2"):
        return
    c2s = configs.c2s()
    A2, B2 = (torch.from_numpy(c2s["buffers"][n].view(np.int32)).cuda() for n in ("A", "B"))
    yield "c2s", c2s["ir"], c2s.get("min_blocks", 0), [A2, B2, torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")]
    if os.environ.get("ONLY_C2S"):
        return
    c3 = configs.c3(**configs.BENCH_C3)
    X = torch.from_numpy(c3["buffers"]["X"].view(np.int32)).cuda()
    yield "c3", c3["ir"], 0, [X, torch.zeros(c3["W"] * c3["H"], dtype=torch.int32, device="cuda")]
    c4 = configs.c4a(1 << 28, grid=1)
    K, S = (torch.from_numpy(c4["buffers"][n].view(np.int32)).cuda() for n in ("keys", "starts"))
    yield "c4a", c4["ir"], 0, [K, S, torch.zeros(256 * 2048, dtype=torch.int32, device="cuda")]


def main(trials):
    s = torch.cuda.Stream()
    print("| config | mode | T0 ms | device overhead per cycle (p50 / p90) µs | kernel + resume ms (p50) | host drain -> resume launch µs (p50) |")
    print("|---|---|---|---|---|---|")
    for name, ir_text, mb, bufs in setups():
        for mname, mode in (("CTXBack", cb.MODE_CTXBACK), ("FULL_HW", cb.MODE_FULL_HW)):
            prog = cb.Program(ir_text, poll_policy=cb.POLL_EXPLICIT, mode=mode, min_blocks_per_sm=mb)
            grid = prog.persistent_grid()
            if name == "c2" and os.environ.get("C2_GRID"):   # e.g. 256: 4 tiles per block, balanced
                grid = int(os.environ["C2_GRID"])
            if name == "c4a":
                bufs[2] = torch.zeros(256 * grid, dtype=torch.int32, device="cuda")
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            t0s = []
            for i in range(6):
                bufs[len(bufs) - 1].zero_()
                run = prog.launch(grid, bufs, [], ctx, s)
                run.wait()
                if i:
                    t0s.append(run.launch_ms())
                del run
            T0 = float(np.median(t0s))
            out_i = len(bufs) - 1
            ref = bufs[out_i].clone()
            ov, tot, gaps = [], [], []
            for f in np.random.default_rng(7).uniform(0.1, 0.9, trials):
                bufs[out_i].zero_()
                torch.cuda.synchronize()
                run = prog.launch(grid, bufs, [], ctx, s)
                bench.spin_until(time.perf_counter() + f * T0 / 1e3)
                st = run.preempt(None)
                if not st["warps_preempted"]:
                    run.wait()
                    del run
                    continue
                t_drain = time.perf_counter()
                k1 = run.launch_ms()
                bench.evict_l2(s)
                t_call = time.perf_counter()
                run.resume(s)
                run.wait()
                k2 = run.launch_ms()
                torch.cuda.synchronize()
                assert torch.equal(bufs[out_i], ref), (name, mname, f)
                ov.append((k1 + k2 - T0) * 1e3)
                tot.append(k1 + k2)
                gaps.append((t_call - t_drain) * 1e6)
                del run
            print(f"| {name} | {mname} | {T0:.3f} | {np.median(ov):.1f} / {np.percentile(ov, 90):.1f} | "
                  f"{np.median(tot):.3f} | {np.median(gaps):.1f} |", flush=True)


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 15)
