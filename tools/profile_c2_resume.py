"""C2's in-situ resume for ncu: the 4096^3 SGEMM on its persistent grid
(296 x 256), every warp preempted at poll visit K (default: its last one; forced mode: under ncu a
flag raised by a stream memory op lands only after the serialised victim),
256 MiB written to evict L2, then the resume kernel restores every warp's
context (69 values + 3 scalars, 8844 B) and runs to completion.
python tools/profile_c2_resume.py [mode=0|3] [K|last]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

mode = int(sys.argv[1]) if len(sys.argv) > 1 else 0
K = sys.argv[2] if len(sys.argv) > 2 else "last"
cfg = configs.c2()
prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode, debug=cb.DEBUG_FORCED, min_blocks_per_sm=2)
bps, nsm = prog.occupancy()
grid = bps * nsm
nw = grid * 8
dA = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
dB = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
dC = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
scratch = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
if K == "last":
    # every warp at its last poll visit (its last tile's last k-iteration), so
    # the resume kernel is the restore plus one iteration and the C tile store
    ntiles = (4096 // 128) ** 2
    tiles = np.array([len(range(b, ntiles, grid)) for b in range(grid)])
    targets = np.repeat(tiles * (4096 // 4) - 1, 8).astype(np.uint32)
else:
    targets = np.full(nw, int(K), np.uint32)
run = prog.launch(grid, [dA, dB, dC], [], ctx, forced=targets)
assert not run.wait()
pb, hb, ntb = run.context_bytes()
scratch.fill_(7)                                 # evict the context from L2
torch.cuda.synchronize()
run.resume(forced=np.full(nw, cb.NEVER, np.uint32))
assert run.wait()
print(f"mode {mode} grid {grid} context {pb} B payload + {hb} B headers over {ntb} TBs; "
      f"resume span {run.resume_stats()['resume_us']:.2f} us, kernel {run.launch_ms() * 1e3:.1f} us")
