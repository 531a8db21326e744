"""CTXB_OSRB_SMEM vs register OSRB slots on C4a (the config with an OSRB
backup): registers per thread, uninterrupted kernel time, preemption routines
and resume.  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def main():
    cfg = configs.c4a(1 << 28, grid=1)
    k = torch.from_numpy(cfg["buffers"]["keys"].view(np.int32)).cuda()
    st = torch.from_numpy(cfg["buffers"]["starts"].view(np.int32)).cuda()
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    rows = ["| OSRB slot | regs | kernel ms (median of 7) | routines µs p50 | resume µs p50 (gathered) | preempted |",
            "|---|---|---|---|---|---|"]
    for name, fl in (("register", 0), ("shared memory", cb.OSRB_SMEM), ("register lanes", cb.OSRB_LANES)):
        prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT,
                          flags=cb.ALL | cb.SYNC_POLL | cb.GATHER_RESUME | fl)
        bps, nsm = prog.occupancy()
        grid = bps * nsm
        h = torch.zeros(256 * grid, dtype=torch.int32, device="cuda")
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        ts = []
        for _ in range(7):
            run = prog.launch(grid, [k, st, h], [], ctx, s)
            run.wait()
            ts.append(run.launch_ms())
            del run
        T = float(np.median(ts))
        lat, res = [], []
        for fr in np.random.default_rng(3).uniform(0.1, 0.9, 9):
            run = prog.launch(grid, [k, st, h], [], ctx, s)
            t0 = time.perf_counter()
            while time.perf_counter() < t0 + fr * T / 1e3:
                pass
            x = run.preempt(ctrl)
            if x["warps_preempted"]:
                lat.append(x["latency_us"])
                run.resume(s)
                while not run.wait():
                    run.resume(s)
                res.append(run.resume_stats()["resume_us"])
            del run
        rows.append(f"| {name} | {prog.info['num_regs']} | {T:.3f} | {np.median(lat):.2f} | {np.median(res):.2f} | "
                    f"{len(lat)}/9 |")
        print(rows[-1], flush=True)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
