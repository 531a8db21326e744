"""Poll-site cost of C3 (stencil) and C4b (BFS) against the same generated
kernel without polls, over the poll-placement knobs: rows per loop iteration
(C3), which sites (C4b), flag word vs replicas, load_every; plus the routines
span of flag preemptions (the latency side of the trade-off).
Usage: python tools/poll_cost_study.py c3|c4b [trials]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
# SIGNAL=watcher: the preemptions go through CTXB_WATCHER + CTXB_DRAIN_NOTICE (the bench's path)
SIG = (cb.WATCHER | cb.DRAIN_NOTICE) if os.environ.get("SIGNAL") == "watcher" else 0


def timed(prog, grid, bufs, uni=(), reps=7):
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    ts = []
    for i in range(reps + 1):
        run = prog.launch(grid, bufs, list(uni), ctx, s)
        run.wait()
        if i:
            ts.append(run.launch_ms())
        del run
    return float(np.median(ts)), ctx


def routines(prog, grid, bufs, ctx, T, trials, uni=()):
    lats = []
    for f in np.random.default_rng(3).uniform(0.1, 0.9, trials):
        run = prog.launch(grid, bufs, list(uni), ctx, s)
        t0 = time.perf_counter()
        while time.perf_counter() < t0 + f * T / 1e3:
            pass
        st = run.preempt(ctrl)
        if st["warps_preempted"]:
            lats.append(st["latency_us"])
            run.resume(s)
        run.wait()
        del run
    return float(np.median(lats)) if lats else float("nan")


def c3(trials):
    base = configs.c3()
    X = torch.from_numpy(base["buffers"]["X"].view(np.int32)).cuda()
    Y = torch.zeros(base["W"] * base["H"], dtype=torch.int32, device="cuda")
    print("| rows/iter | polls | flag | load_every | kernel ms | no-polls ms | overhead | routines us |")
    print("|---|---|---|---|---|---|---|---|")
    for R in (2, 4, 8, 16):
        for polls in ("both", "end"):
            txt = configs.c3_ir(rows_per_iter=R, polls=polls)
            np_prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_POLLS)
            bps, nsm = np_prog.occupancy()
            grid = bps * nsm
            t0, _ = timed(np_prog, grid, [X, Y])
            for fname, fl in (("word", 0), ("replicas", cb.FLAG_REPLICAS)):
                for le in (1, 4):
                    prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | fl, load_every=le)
                    g = min(grid, prog.occupancy()[0] * nsm)
                    t, ctx = timed(prog, g, [X, Y])
                    lat = routines(prog, g, [X, Y], ctx, t, trials)
                    print(f"| {R} | {polls} | {fname} | {le} | {t:.3f} | {t0:.3f} | {100 * (t / t0 - 1):.1f} % | {lat:.2f} |",
                          flush=True)


def c4b(trials):
    rp, ci = configs.c4b_graph()
    n = len(rp) - 1
    d_rp = torch.from_numpy(rp.view(np.int32)).cuda()
    d_ci = torch.from_numpy(ci.view(np.int32)).cuda()
    fronts = [torch.zeros(n + 1, dtype=torch.int32, device="cuda") for _ in range(2)]
    dist = torch.empty(n, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    want = torch.from_numpy(configs.bfs_reference(rp, ci).view(np.int32)).cuda()

    def bfs(prog, grid, ctx, plevel=None, delay=0.0):
        dist.fill_(-1)
        dist[0] = 0
        fronts[0][0] = 0
        nf, lvl, tot, lat, sizes = 1, 0, 0.0, None, []
        while nf:
            cnt.zero_()
            torch.cuda.synchronize()
            run = prog.launch(grid, [d_rp, d_ci, fronts[lvl % 2], dist, fronts[(lvl + 1) % 2], cnt], [nf, lvl + 1],
                              ctx, s)
            if lvl == plevel:
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + delay:
                    pass
                st = run.preempt(ctrl)
                if st["warps_preempted"]:
                    lat = st["latency_us"]
                    run.resume(s)
                run.wait()
            else:
                run.wait()
                tot += run.launch_ms()
            sizes.append(run.launch_ms())
            del run
            nf = int(cnt.item())
            lvl += 1
        assert torch.equal(dist, want)
        return tot, lat, sizes

    print("| polls | flag | load_every | BFS ms | no-polls ms | overhead | routines us |")
    print("|---|---|---|---|---|---|---|")
    base = cb.Program(configs.c4b_ir(), poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_POLLS)
    bps, nsm = base.occupancy()
    grid = bps * nsm
    ctx = torch.empty(base.context_capacity(grid), dtype=torch.uint8, device="cuda")
    bfs(base, grid, ctx)
    t0 = float(np.median([bfs(base, grid, ctx)[0] for _ in range(5)]))
    variants = [(p, f, str(le)) for p in ("both", "vertex", "edge") for f in ("word", "replicas") for le in (1, 4)]
    if os.environ.get("C4B_VARIANTS"):      # e.g. "edge:replicas:1,edge:replicas:2"
        variants = [tuple(v.split(":")) for v in os.environ["C4B_VARIANTS"].split(",")]   # polls:flag:K[:sync]
    for var in variants:
        polls, fname, le = var[0], var[1], int(var[2])
        txt = configs.c4b_ir(polls)
        fl = {"word": 0, "replicas": cb.FLAG_REPLICAS}[fname] | (cb.SYNC_POLL if len(var) > 3 else 0)
        if len(var) > 3:
            fname += " sync"
        if True:
            if True:
                prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | fl | SIG, load_every=le)
                grid = prog.persistent_grid()      # room for the watcher warp (a block waiting for it doubles the tail)
                ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
                _, _, sizes = bfs(prog, grid, ctx)
                big = int(np.argmax(sizes))
                T = float(np.median([bfs(prog, grid, ctx)[0] for _ in range(5)]))
                lats = [bfs(prog, grid, ctx, big, f * sizes[big] / 1e3)[1]
                        for f in np.random.default_rng(4).uniform(0.1, 0.9, trials)]
                lats = [x for x in lats if x is not None]
                print(f"| {polls} | {fname} | {le} | {T:.3f} | {t0:.3f} | {100 * (T / t0 - 1):.1f} % | "
                      f"{np.median(lats) if lats else float('nan'):.2f} |", flush=True)


if __name__ == "__main__":
    which = sys.argv[1] if len(sys.argv) > 1 else "c3"
    trials = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    {"c3": c3, "c4b": c4b}[which](trials)
