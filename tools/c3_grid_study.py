"""C3 (bench placement) on the default signal path: does the grid (resident
blocks per SM) or the flag word the sites poll change the preemption?
Round 2: recomputing the context pointers in the save routines
cut C3's kernel from 40 to 32 registers, so its persistent grid grew from
6 x 148 to 8 x 148 blocks and the bench's C3 routines span grew (3.5 -> 4.7
us).  Rows: flags x grid; kernel ms (polled / no polls, same grid), routines,
host latency and L2-cold resume medians over flag preemptions at random times.
Usage: python tools/c3_grid_study.py [trials]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def main(trials=15):
    cfg = configs.c3(**configs.BENCH_C3)
    W, H = cfg["W"], cfg["H"]
    X = torch.from_numpy(cfg["buffers"]["X"].view(np.int32)).cuda()
    Y = torch.zeros(W * H, dtype=torch.int32, device="cuda")
    want = torch.from_numpy(configs.c3_numpy_reference(cfg["buffers"]["X"], W, H).view(np.int32)).cuda()
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    NA = cb.DEBUG_NO_AUTO_SIGNAL
    sig = cb.WATCHER | cb.DRAIN_NOTICE
    variants = [("sync (default)", sig | cb.SYNC_POLL), ("sync + replicas", sig | cb.SYNC_POLL | cb.FLAG_REPLICAS),
                ("pipelined + replicas", sig | cb.FLAG_REPLICAS)]
    print("| flags | mode | grid | kernel ms | no-polls ms | overhead | routines us | host us | resume us |")
    print("|---|---|---|---|---|---|---|---|---|")
    for vname, fl in variants:
        for mode_name, mode in (("CTXBack", cb.MODE_CTXBACK), ("FULL_HW", cb.MODE_FULL_HW)):
            if mode == cb.MODE_FULL_HW and vname != "sync (default)":
                continue
            prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode, flags=cb.ALL | fl, debug=NA)
            nop = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode,
                             flags=cb.ALL | (fl & ~cb.WATCHER), debug=NA | cb.DEBUG_NO_POLLS)
            g_full = prog.persistent_grid()
            nsm = prog.occupancy()[1]
            for grid in sorted({g_full, 6 * nsm}):
                ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
                ts = {"p": [], "n": []}
                for i in range(8):
                    for k, p in (("p", prog), ("n", nop)):
                        run = p.launch(grid, [X, Y], [], ctx, s)
                        run.wait()
                        if i:
                            ts[k].append(run.launch_ms())
                        del run
                T = float(np.median(ts["p"]))
                rt, host, res = [], [], []
                for f in np.random.default_rng(5).uniform(0.05, 0.95, trials):
                    Y.zero_()
                    torch.cuda.synchronize()
                    run = prog.launch(grid, [X, Y], [], ctx, s)
                    bench.spin_until(time.perf_counter() + f * T / 1e3)
                    st = run.preempt(None)
                    if st["warps_preempted"]:
                        rt.append(st["latency_us"])
                        host.append(st["host_us"])
                        bench.evict_l2(s)
                        run.resume(s)
                        run.wait()
                        res.append(run.resume_stats()["resume_us"])
                    run.wait()
                    torch.cuda.synchronize()
                    assert torch.equal(Y, want), (vname, mode_name, grid)
                    del run
                n = float(np.median(ts["n"]))
                print(f"| {vname} | {mode_name} | {grid} | {T:.4f} | {n:.4f} | {100 * (T / n - 1):.1f} % | "
                      f"{np.median(rt):.2f} | {np.median(host):.2f} | {np.median(res):.2f} |", flush=True)


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 15)
