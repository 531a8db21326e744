"""Diagnostic: count C2's tile-loop and k-loop iterations (atomic counters
added to the IR) in an uninterrupted run and in a run preempted at every
warp's poll visit K and resumed (forced mode), per mode.
python tools/resume_count_probe.py [K]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 1
ir = configs.c2()["ir"]
ir = ir.replace(".buffer wo C", ".buffer wo C\n.buffer rw cnt").replace(".vregs 104", ".vregs 106")
ir = ir.replace("init:\n", "init:\n  setp.eq.u v104, %laneid, 0\n", 1)
ir = ir.replace("store:\n", "store:\n  @v104 atom.add _, cnt[0], 1\n", 1)
ir = ir.replace("  poll\n", "  @v104 atom.add _, cnt[1], 1\n  poll\n", 1)
cfg = configs.c2()
dA = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
dB = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
dC = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
cnt = torch.zeros(64, dtype=torch.int32, device="cuda")
for mname, mode in (("CTXBack", 0), ("FULL_IR", 2)):
    prog = cb.Program(ir, poll_policy=cb.POLL_EXPLICIT, mode=mode, debug=cb.DEBUG_FORCED, min_blocks_per_sm=2,
                      flags=cb.ALL)
    grid = prog.persistent_grid()
    nw = grid * 8
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    never = np.full(nw, cb.NEVER, np.uint32)
    cnt.zero_()
    run = prog.launch(grid, [dA, dB, dC, cnt], [], ctx, forced=never)
    assert run.wait()
    t0 = run.launch_ms()
    u = cnt[:2].cpu().tolist()
    ref = dC.clone()
    dC.zero_()
    cnt.zero_()
    run = prog.launch(grid, [dA, dB, dC, cnt], [], ctx, forced=np.full(nw, K, np.uint32))
    assert not run.wait()
    a = cnt[:2].cpu().tolist()
    run.resume(forced=never)
    assert run.wait()
    t1 = run.launch_ms()
    b = cnt[:2].cpu().tolist()
    torch.cuda.synchronize()
    print(f"{mname}: uninterrupted tiles x warps {u[0]} k-iterations x warps {u[1]} ({t0:.2f} ms); "
          f"preempted at {K}: {a}; after resume {b} ({t1:.2f} ms); C equal: {bool(torch.equal(dC, ref))}", flush=True)
