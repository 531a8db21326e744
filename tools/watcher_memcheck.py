"""A small flag preemption on the library's default path (DESIGN.md 8q:
CTXB_WATCHER + drain notice + the cost model's poll test, gathered resume for
atomics), for compute-sanitizer: C2 at 256^3, C3 at 2048 x 1024 and C4a at
2^16 keys, preempted by the watcher (no memop fallback), resumed, compared
with the uninterrupted run."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def run_case(txt, bufs, out_i, extra=0, mb=0):
    prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | extra, min_blocks_per_sm=mb)
    assert prog.info["flags"] & (cb.WATCHER | cb.DRAIN_NOTICE) == cb.WATCHER | cb.DRAIN_NOTICE
    grid = prog.persistent_grid()
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    bufs[out_i].zero_()
    run = prog.launch(grid, bufs, [], ctx, s)
    assert run.wait()
    ref = bufs[out_i].clone()
    T = run.launch_ms() / 1e3
    npre = 0
    for fr in (0.2, 0.5):
        bufs[out_i].zero_()
        torch.cuda.synchronize()
        run = prog.launch(grid, bufs, [], ctx, s)
        t0 = time.perf_counter()
        while time.perf_counter() < t0 + fr * T:
            pass
        st = run.preempt(None)                      # the watcher alone
        npre += st["warps_preempted"]
        while not run.finished:
            run.resume(s)
            run.wait()
        torch.cuda.synchronize()
        assert torch.equal(bufs[out_i], ref)
    return npre


c2 = configs.c2(256, 256, 256)
a, b = (torch.from_numpy(c2["buffers"][n].view(np.int32)).cuda() for n in ("A", "B"))
print("c2 preempted warps:", run_case(c2["ir"], [a, b, torch.zeros(256 * 256, dtype=torch.int32, device="cuda")], 2,
                                      mb=c2["min_blocks"]))
c3 = configs.c3(2048, 1024, 64, **configs.BENCH_C3)
x = torch.from_numpy(c3["buffers"]["X"].view(np.int32)).cuda()
print("c3 preempted warps:", run_case(c3["ir"], [x, torch.zeros(2048 * 1024, dtype=torch.int32, device="cuda")], 1))
c4 = configs.c4a(1 << 16, grid=1)
k = torch.from_numpy(c4["buffers"]["keys"].view(np.int32)).cuda()
st = torch.from_numpy(c4["buffers"]["starts"].view(np.int32)).cuda()
print("c4a preempted warps:", run_case(c4["ir"], [k, st, torch.zeros(256 * 2048, dtype=torch.int32, device="cuda")], 2,
                                       ))
print("ok")
