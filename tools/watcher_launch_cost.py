"""What a CTXB_WATCHER launch costs when nothing is preempted: C4b's BFS (22
short launches, one per level) and C2 (one long launch), uninterrupted, with
the memop path (nothing extra at launch) vs the watcher (+ drain notice):
host wall time of the whole job (launches, per-level count read-back) and the
summed kernel times.  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def bfs_job(prog, grid, bufs, ctx, s):
    d_rp, d_ci, fronts, dist, cnt = bufs
    dist.fill_(-1)
    dist[0] = 0
    fronts[0][0] = 0
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    nf, lvl, ktime = 1, 0, 0.0
    while nf:
        cnt.zero_()
        run = prog.launch(grid, [d_rp, d_ci, fronts[lvl % 2], dist, fronts[(lvl + 1) % 2], cnt], [nf, lvl + 1], ctx, s)
        run.wait()
        ktime += run.launch_ms()
        del run
        nf = int(cnt.item())
        lvl += 1
    return (time.perf_counter() - t0) * 1e3, ktime, lvl


def main():
    s = torch.cuda.Stream()
    rp, ci = configs.c4b_graph()
    n = len(rp) - 1
    bufs = (torch.from_numpy(rp.view(np.int32)).cuda(), torch.from_numpy(ci.view(np.int32)).cuda(),
            [torch.zeros(n + 1, dtype=torch.int32, device="cuda") for _ in range(2)],
            torch.empty(n, dtype=torch.int32, device="cuda"), torch.zeros(1, dtype=torch.int32, device="cuda"))
    c2 = configs.c2()
    a = torch.from_numpy(c2["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(c2["buffers"]["B"].view(np.int32)).cuda()
    c = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    print("| job | signal path | wall ms (median of 9) | summed kernel ms | launches |")
    print("|---|---|---|---|---|")
    for name, fl in (("memop", 0), ("watcher + notice", cb.WATCHER | cb.DRAIN_NOTICE)):
        prog = cb.Program(configs.c4b_ir(configs.BENCH_C4B_POLLS), poll_policy=cb.POLL_EXPLICIT,
                          flags=cb.ALL | cb.FLAG_REPLICAS | fl)
        grid = prog.persistent_grid()
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        bfs_job(prog, grid, bufs, ctx, s)
        r = [bfs_job(prog, grid, bufs, ctx, s) for _ in range(9)]
        print(f"| C4b BFS 2^22 | {name} | {np.median([x[0] for x in r]):.3f} | {np.median([x[1] for x in r]):.3f} | "
              f"{r[0][2]} |", flush=True)
    for name, fl in (("memop", 0), ("watcher + notice", cb.WATCHER | cb.DRAIN_NOTICE)):
        prog = cb.Program(c2["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, flags=cb.ALL | fl)
        grid = prog.persistent_grid()
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        w, k = [], []
        for i in range(10):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            run = prog.launch(grid, [a, b, c], [], ctx, s)
            run.wait()
            if i:
                w.append((time.perf_counter() - t0) * 1e3)
                k.append(run.launch_ms())
            del run
        print(f"| C2 SGEMM 4096^3 | {name} | {np.median(w):.3f} | {np.median(k):.3f} | 1 |", flush=True)


if __name__ == "__main__":
    main()
