"""Run the C2 kernel once uninterrupted (for ncu): python tools/run_c2_once.py [polls|nopolls] [size]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

variant = sys.argv[1] if len(sys.argv) > 1 else "polls"
size = int(sys.argv[2]) if len(sys.argv) > 2 else 4096
placement = os.environ.get("POLLS", "iter")
depth = int(os.environ.get("DEPTH", "1"))
dbg = cb.DEBUG_NO_POLLS if variant == "nopolls" else (cb.DEBUG_FORCED if variant == "forced" else 0)
mb = int(os.environ.get("MINB", "0"))
prog = cb.Program(configs.c2_ir(size, size, size, polls=placement), poll_policy=cb.POLL_EXPLICIT, debug=dbg,
                  flag_depth=depth, min_blocks_per_sm=mb)
bps, nsm = prog.occupancy()
grid = bps * nsm
r = np.random.default_rng(0)
dA = torch.from_numpy(r.uniform(-1, 1, size * size).astype(np.float32).view(np.int32)).cuda()
dB = torch.from_numpy(r.uniform(-1, 1, size * size).astype(np.float32).view(np.int32)).cuda()
dC = torch.zeros(size * size, dtype=torch.int32, device="cuda")
ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
nw = grid * 8
for i in range(int(os.environ.get("REPS", "2"))):
    run = prog.launch(grid, [dA, dB, dC], [], ctx,
                      forced=np.full(nw, cb.NEVER, np.uint32) if variant == "forced" else None)
    run.wait()
    print(variant, "minb", mb, placement, "D", depth, "ms", round(run.launch_ms(), 3), "regs", prog.info["num_regs"],
          prog.info["num_regs_resume"], "grid", grid)
