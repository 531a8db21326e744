"""Two watched runs (C3, C2) in flight at once, step by step with a
faulthandler watchdog logging to gpurun_out/conc.log: the reproduction of
the module-load deadlock fixed in round 2."""
import faulthandler, sys, time, os
sys.path.insert(0, '/root/repo'); sys.path.insert(0, '/root/repo/tests')
log = open('/root/repo/gpurun_out/conc.log', 'w', buffering=1)
faulthandler.dump_traceback_later(60, exit=True, file=log)
import numpy as np, torch
import paper_conf_ipps_jiw21_b200 as cb
from workloads import configs
from gpu_helpers import to_dev
def P(*a): print(*a, file=log, flush=True)
c3 = configs.c3(2048, 2048, 64, **configs.BENCH_C3)
x = to_dev(c3["buffers"]["X"]); y = torch.zeros(2048 * 2048, dtype=torch.int32, device="cuda")
c2 = configs.c2(1024, 1024, 1024)
a, b = to_dev(c2["buffers"]["A"]), to_dev(c2["buffers"]["B"]); c = torch.zeros(1024 * 1024, dtype=torch.int32, device="cuda")
fl = cb.ALL | cb.WATCHER | cb.DRAIN_NOTICE
p3 = cb.Program(c3["ir"], poll_policy=cb.POLL_EXPLICIT, flags=fl)
p2 = cb.Program(c2["ir"], poll_policy=cb.POLL_EXPLICIT, flags=fl, min_blocks_per_sm=2)
P("compiled")
g3, g2 = 32, 16
ctx3 = torch.zeros(p3.context_capacity(g3), dtype=torch.uint8, device="cuda")
ctx2 = torch.zeros(p2.context_capacity(g2), dtype=torch.uint8, device="cuda")
s3, s2 = torch.cuda.Stream(), torch.cuda.Stream()
r3 = p3.launch(g3, [x, y], [], ctx3, s3); P("launched 3")
P("wait3", r3.wait())
r2 = p2.launch(g2, [a, b, c], [], ctx2, s2); P("launched 2")
P("wait2", r2.wait())
r3, r2 = p3.launch(g3, [x, y], [], ctx3, s3), p2.launch(g2, [a, b, c], [], ctx2, s2); P("launched both")
P("wait3", r3.wait()); P("wait2", r2.wait())
P("done")
ref3, ref2 = y.clone(), c.clone()
for delay in (20e-6, 200e-6):
    y.zero_(); c.zero_(); torch.cuda.synchronize()
    r3, r2 = p3.launch(g3, [x, y], [], ctx3, s3), p2.launch(g2, [a, b, c], [], ctx2, s2)
    P("launched", delay)
    t0 = time.perf_counter()
    while time.perf_counter() < t0 + delay:
        pass
    st3 = r3.preempt(None); P("preempted 3", st3["warps_preempted"], st3["host_us"])
    st2 = r2.preempt(None); P("preempted 2", st2["warps_preempted"], st2["host_us"])
    for nm, r, s in (("3", r3, s3), ("2", r2, s2)):
        k = 0
        while not r.finished:
            r.resume(s); P("resumed", nm, k); r.wait(); P("waited", nm, k); k += 1
    torch.cuda.synchronize()
    P("equal", torch.equal(y, ref3), torch.equal(c, ref2))
P("all done")
