"""C2: drain latency and signal->drained (CUDA events) with and without the
save stub's __threadfence (CTXB_DEBUG_FENCE_STAMPS = 32)."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

cfg = configs.c2()
bufs = [torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda(),
        torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda(),
        torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")]
s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
for name, mode, dbg in (("ctxback fence", 0, 32), ("ctxback nofence", 0, 0), ("full_hw fence", 3, 32),
                        ("full_hw nofence", 3, 0)):
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode, debug=dbg, min_blocks_per_sm=2)
    bps, nsm = prog.occupancy()
    grid = bps * nsm
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    run = prog.launch(grid, bufs, [], ctx, s)
    run.wait()
    T = run.launch_ms() / 1e3
    del run
    lat, sig, res = [], [], []
    rng = np.random.default_rng(1)
    for i in range(15):
        run = prog.launch(grid, bufs, [], ctx, s)
        t0 = time.perf_counter()
        while time.perf_counter() < t0 + rng.uniform(0.1, 0.9) * T:
            pass
        st = run.preempt(ctrl)
        if st["warps_preempted"]:
            lat.append(st["latency_us"])
            sig.append(st["signal_to_drained_us"])
            run.resume(s)
            run.wait()
            res.append(run.resume_stats()["resume_us"])
        del run
    print(f"{name:18s} drain {np.median(lat):.2f} us  signal->drained {np.median(sig):.2f} us  resume {np.median(res):.2f} us")
