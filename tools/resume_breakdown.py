"""Per-warp breakdown of resume time (C3 or C2): entry spread vs per-warp restore."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "c3"
gather = cb.GATHER_RESUME if "gather" in sys.argv[2:] else 0
if which == "c3":
    cfg = configs.c3()
    mk = lambda: [torch.from_numpy(cfg["buffers"]["X"].view(np.int32)).cuda(),  # noqa: E731
                  torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")]
    mb = 0
elif which == "c4a":
    cfg = configs.c4a(1 << 28, grid=1)
    keys_t = torch.from_numpy(cfg["buffers"]["keys"].view(np.int32)).cuda()
    st_t = torch.from_numpy(cfg["buffers"]["starts"].view(np.int32)).cuda()
    mk = lambda: [keys_t, st_t, torch.zeros(256 * 148 * 8, dtype=torch.int32, device="cuda")]  # noqa: E731
    mb = 0
else:
    cfg = configs.c2()
    mk = lambda: [torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda(),  # noqa: E731
                  torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda(),
                  torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")]
    mb = 2
bufs = mk()
s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
for name, mode in (("ctxback", 0), ("full_hw", 3), ("full_ir", 2), ("live", 1)):
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode, min_blocks_per_sm=mb, flags=cb.ALL | gather)
    bps, nsm = prog.occupancy()
    grid = bps * nsm
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    run = prog.launch(grid, bufs, [], ctx, s)
    run.wait()
    T = run.launch_ms() / 1e3
    del run
    for trial in range(3):
        run = prog.launch(grid, bufs, [], ctx, s)
        t0 = time.perf_counter()
        while time.perf_counter() < t0 + 0.5 * T:
            pass
        st = run.preempt(ctrl)
        h = run.headers().copy()
        pre = (h[:, 2] == 1) & (h[:, 3] == 1)
        run.resume(s)
        run.wait()
        rs = run.resume_stats()
        ms = run.launch_ms()
        stp = run.stamps()[pre]
        ent, site = stp[:, 2].astype(np.int64), stp[:, 3].astype(np.int64)
        if which in ("c4a", "c4b") or gather:
            order = np.argsort(ent)
            print("   entry quantiles (us from first):", np.percentile((ent - ent.min()) / 1e3, [0, 50, 90, 99, 100]).round(2),
                  "site quantiles:", np.percentile((site - ent.min()) / 1e3, [0, 50, 90, 99, 100]).round(2),
                  "occupancy", prog.occupancy(), "regs", prog.info["num_regs"], prog.info["num_regs_resume"])
        dur = (site - ent) / 1e3
        print(f"{name:8s} grid {grid} preempted {pre.sum()} lat {st['latency_us']:.2f} resume {rs['resume_us']:.2f} us "
              f"kernel {ms * 1e3:.1f} us | entry spread {(ent.max() - ent.min()) / 1e3:.2f} us, per-warp restore "
              f"p50 {np.median(dur):.2f} p90 {np.percentile(dur, 90):.2f} max {dur.max():.2f} us | save: seen spread "
              f"{(stp[:, 0].max() - stp[:, 0].min()) / 1e3:.2f} per-warp save p50 "
              f"{np.median((stp[:, 1].astype(np.int64) - stp[:, 0].astype(np.int64)) / 1e3):.2f} us")
        del run
