"""Is C2's resume kernel slower than its normal kernel on the same work?
Forced mode: one uninterrupted launch (ctxb_run), then a launch preempted at
every warp's poll visit K (default 1: almost all work is left), then its
resume (ctxb_resume runs the rest).  Prints the kernel times; under ncu
(`-k regex:ctxb_ -c 3`) the three launches are the ones to compare.
python tools/resume_speed_probe.py [K] [mode] [flags-extra]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 1
mode = int(sys.argv[2]) if len(sys.argv) > 2 else 0
cfg = configs.c2()
prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode, debug=cb.DEBUG_FORCED, min_blocks_per_sm=2)
grid = prog.persistent_grid()
nw = grid * 8
dA = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
dB = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
dC = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
never = np.full(nw, cb.NEVER, np.uint32)
ts = []
for i in range(3):
    run = prog.launch(grid, [dA, dB, dC], [], ctx, forced=never)
    assert run.wait()
    ts.append(run.launch_ms())
ref = dC.clone()
dC.zero_()
run = prog.launch(grid, [dA, dB, dC], [], ctx, forced=np.full(nw, K, np.uint32))
assert not run.wait()
t1 = run.launch_ms()
run.resume(forced=never)
assert run.wait()
t2 = run.launch_ms()
torch.cuda.synchronize()
assert torch.equal(dC, ref)
print(f"grid {grid}: uninterrupted {np.median(ts):.3f} ms; preempted at visit {K}: {t1:.3f} ms + resume {t2:.3f} ms "
      f"= {t1 + t2:.3f} ms (+{(t1 + t2 - np.median(ts)) * 1e3:.0f} us)")
