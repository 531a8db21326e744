"""C4b detection with the memop vs the watcher signal (largest level, 4
preemptions each): routines span, first-seen -> median / p99 / last-seen
spread, host latency, watcher raise -> first warp (profiles/r02_poll_placement.md)."""
import sys, time, numpy as np, torch
sys.path.insert(0, '/root/repo')
import paper_conf_ipps_jiw21_b200 as cb
from workloads import configs
rp, ci = configs.c4b_graph(); n = len(rp) - 1
d_rp = torch.from_numpy(rp.view(np.int32)).cuda(); d_ci = torch.from_numpy(ci.view(np.int32)).cuda()
fronts = [torch.zeros(n + 1, dtype=torch.int32, device="cuda") for _ in range(2)]
dist = torch.empty(n, dtype=torch.int32, device="cuda"); cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
for name, fl in (("memop", 0), ("watcher", cb.WATCHER | cb.DRAIN_NOTICE), ("watcher-nonotice", cb.WATCHER)):
    prog = cb.Program(configs.c4b_ir("edge"), poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | cb.FLAG_REPLICAS | fl)
    grid = prog.persistent_grid()
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    for trial in range(4):
        dist.fill_(-1); dist[0] = 0; fronts[0][0] = 0
        nf, lvl, out = 1, 0, []
        while nf:
            cnt.zero_(); torch.cuda.synchronize()
            run = prog.launch(grid, [d_rp, d_ci, fronts[lvl % 2], dist, fronts[(lvl + 1) % 2], cnt], [nf, lvl + 1], ctx, s)
            if lvl == 6:
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + 100e-6: pass
                st = run.preempt(ctrl)
                if st["warps_preempted"]:
                    h = run.headers(); pre = (h[:, 2] == 1) & (h[:, 3] == 1)
                    stp = run.stamps()[pre].astype(np.int64)
                    seen = (stp[:, 0] - stp[:, 0].min()) / 1e3; saved = (stp[:, 1] - stp[:, 0].min()) / 1e3
                    w = run.watcher_stamp()
                    out.append((lvl, st["warps_preempted"], round(st["latency_us"], 2), round(st["host_us"], 2),
                                np.percentile(seen, [50, 90, 99, 100]).round(2).tolist(),
                                np.percentile(saved, [50, 99, 100]).round(2).tolist(),
                                round((stp[:, 0].min() - w) / 1e3, 2) if w else None))
                    run.resume(s)
                run.wait()
            else:
                run.wait()
            del run
            nf = int(cnt.item()); lvl += 1
        print(name, grid, out)
