"""The README quick-start snippet (kept runnable)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch, paper_conf_ipps_jiw21_b200 as cb
from workloads import configs

cfg = configs.c2()                                         # 4096^3 tiled SGEMM IR kernel
prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)   # ctxb_analyze
# defaults: watcher warp + drain notice + synchronous flag test
assert prog.info["flags"] & (cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL) == cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL
grid = prog.persistent_grid()                              # every block resident, room for the watcher
A = torch.from_numpy(cfg["buffers"]["A"].view("int32")).cuda()
B = torch.from_numpy(cfg["buffers"]["B"].view("int32")).cuda()
C = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
run = prog.launch(grid, [A, B, C], [], ctx, s)             # ctxb_launch (+ its watcher warp)
st = run.preempt(None)                                     # ctxb_preempt: the watcher relays the signal,
                                                           # every warp saves and exits
print(st["host_us"], st["latency_us"], run.context_bytes())   # host latency, routines span, bytes
run.resume(s); run.wait()                                  # ctxb_resume: restore, replay, continue
