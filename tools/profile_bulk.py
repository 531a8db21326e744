"""One bulk context save (ctxb_run) and restore (ctxb_resume) of >= 1 GiB through
the generated stubs, for ncu.  python tools/profile_bulk.py [MiB]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

mib = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
prog = cb.Program(configs.bulk_ir(64), poll_policy=cb.POLL_EXPLICIT, mode=cb.MODE_LIVE, debug=cb.DEBUG_FORCED, min_blocks_per_sm=configs.BULK_MIN_BLOCKS)
nw = (mib << 20) // (64 * 128)
grid = nw // 8
nw = grid * 8
out = torch.zeros(256, dtype=torch.int32, device="cuda")
ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
for i in range(int(os.environ.get("REPS", "1"))):
    run = prog.launch(grid, [out], [], ctx, forced=np.zeros(nw, np.uint32))
    assert not run.wait()
    a = run.launch_ms()
    run.resume(forced=np.full(nw, cb.NEVER, np.uint32))
    assert run.wait()
    b = run.launch_ms()
    print(f"save {a:.4f} ms restore {b:.4f} ms payload {nw * 8192} B regs {prog.info['num_regs']}/"
          f"{prog.info['num_regs_resume']}")
