"""C4b (level-synchronous BFS, 2^22 vertices): total kernel time of all
levels, uninterrupted, for the flag-poll variants (one word / replicas x
load_every) against the build without polls; and the routines span of flag
preemptions in the largest level.  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def main():
    rp, ci = configs.c4b_graph()
    n = len(rp) - 1
    want = torch.from_numpy(configs.bfs_reference(rp, ci).view(np.int32)).cuda()
    d_rp = torch.from_numpy(rp.view(np.int32)).cuda()
    d_ci = torch.from_numpy(ci.view(np.int32)).cuda()
    fronts = [torch.zeros(n + 1, dtype=torch.int32, device="cuda") for _ in range(2)]
    dist = torch.empty(n, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    txt = configs.c4b_ir()

    def bfs(prog, grid, ctx, preempt_level=None, delay=0.0):
        dist.fill_(-1)
        dist[0] = 0
        fronts[0][0] = 0
        nf, lvl, tot, lat = 1, 0, 0.0, None
        sizes = []
        while nf:
            cnt.zero_()
            torch.cuda.synchronize()
            run = prog.launch(grid, [d_rp, d_ci, fronts[lvl % 2], dist, fronts[(lvl + 1) % 2], cnt], [nf, lvl + 1],
                              ctx, s)
            if lvl == preempt_level:
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

    rows = ["| variant | BFS kernel ms (all levels) | overhead vs no polls | routines µs p50 (largest level) |",
            "|---|---|---|---|"]
    base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_POLLS)
    bps, nsm = base.occupancy()
    grid = bps * nsm
    ctx = torch.empty(base.context_capacity(grid), dtype=torch.uint8, device="cuda")
    bfs(base, grid, ctx)
    t0 = float(np.median([bfs(base, grid, ctx)[0] for _ in range(5)]))
    for nm, fl in (("one word", 0), ("replicas", cb.FLAG_REPLICAS)):
        for k in (1, 4, 16):
            prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | fl, load_every=k)
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            _, _, sizes = bfs(prog, grid, ctx)
            big = int(np.argmax(sizes))
            T = float(np.median([bfs(prog, grid, ctx)[0] for _ in range(5)]))
            lats = [bfs(prog, grid, ctx, big, f * sizes[big] / 1e3)[1] for f in np.random.default_rng(4).uniform(0.1, 0.9, 7)]
            lats = [x for x in lats if x is not None]
            rows.append(f"| {nm}, load every {k} | {T:.3f} | {100 * (T / t0 - 1):.1f} % | "
                        f"{np.median(lats) if lats else float('nan'):.2f} |")
            print(rows[-1], flush=True)
    print(f"no polls: {t0:.3f} ms")
    print("\n".join(rows))


if __name__ == "__main__":
    main()
