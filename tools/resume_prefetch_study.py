"""A/B of the resume-entry L2 prefetch (default) against CTXB_DEBUG_NO_PREFETCH:
L2-cold in-situ resume of C2 / C3 / C4b (flag at 50 % of T, 256 MiB written
between preempt and resume), CTXBack and FULL_HW; and the bulk restore
kernel's bandwidth.  Usage: python tools/resume_prefetch_study.py [trials]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

trials = int(sys.argv[1]) if len(sys.argv) > 1 else 7
scratch = torch.empty(64 << 20, dtype=torch.int32, device="cuda")


def evict(s):
    with torch.cuda.stream(s):
        scratch.fill_(1)


def c2():
    cfg = configs.c2()
    b = [torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda(),
         torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda(),
         torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")]
    return cfg["ir"], b, 2, {}


def c3():
    cfg = configs.c3(rows_per_iter=2)
    b = [torch.from_numpy(cfg["buffers"]["X"].view(np.int32)).cuda(),
         torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")]
    return cfg["ir"], b, 0, {"load_every": 4}


def study(name, ir_text, bufs, mb, kw):
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    for mode_name, mode in (("ctxback", 0), ("full_hw", 3)):
        for pf_name, dbg in (("prefetch", 0), ("no_prefetch", cb.DEBUG_NO_PREFETCH)):
            prog = cb.Program(ir_text, poll_policy=cb.POLL_EXPLICIT, mode=mode, min_blocks_per_sm=mb, debug=dbg, **kw)
            bps, nsm = prog.occupancy()
            grid = bps * nsm
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            run = prog.launch(grid, bufs, [], ctx, s)
            run.wait()
            T = run.launch_ms() / 1e3
            del run
            res, per, spread, ms = [], [], [], []
            for _ in range(trials):
                run = prog.launch(grid, bufs, [], ctx, s)
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + 0.5 * T:
                    pass
                run.preempt(ctrl)
                h = run.headers().copy()
                pre = (h[:, 2] == 1) & (h[:, 3] == 1)
                if not pre.any():
                    continue
                evict(s)
                run.resume(s)
                run.wait()
                res.append(run.resume_stats()["resume_us"])
                stp = run.stamps()[pre].astype(np.int64)
                per.append(np.median(stp[:, 3] - stp[:, 2]) / 1e3)
                spread.append((stp[:, 2].max() - stp[:, 2].min()) / 1e3)
                del run
            pb = int(h[pre, 1].astype(np.int64).sum())
            print(f"{name:4s} {mode_name:8s} {pf_name:12s} resume p50 {np.median(res):6.2f} us (min {min(res):5.2f})  "
                  f"per-warp p50 {np.median(per):5.2f}  entry spread {np.median(spread):5.2f}  payload {pb / 1e6:5.1f} MB "
                  f"-> {pb / np.median(res) / 1e3:6.0f} GB/s", flush=True)


def bulk(mib=1024, reps=5):
    for pf_name, dbg in (("prefetch", 0), ("no_prefetch", cb.DEBUG_NO_PREFETCH)):
        prog = cb.Program(configs.bulk_ir(64), poll_policy=cb.POLL_EXPLICIT, mode=cb.MODE_LIVE,
                          debug=cb.DEBUG_FORCED | dbg)
        nw = (mib << 20) // 8192
        grid = nw // 8
        out = torch.zeros(256, dtype=torch.int32, device="cuda")
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        t = []
        for i in range(reps + 1):
            run = prog.launch(grid, [out], [], ctx, forced=np.zeros(nw, np.uint32))
            run.wait()
            run.resume(forced=np.full(nw, cb.NEVER, np.uint32))
            run.wait()
            if i:
                t.append(run.launch_ms())
            del run
        by = nw * 8192 + 2 * nw * 16
        print(f"bulk restore {pf_name:12s} {np.median(t):.3f} ms -> {by / np.median(t) / 1e6:.0f} GB/s", flush=True)


if __name__ == "__main__":
    which = sys.argv[2].split(",") if len(sys.argv) > 2 else ["c2", "c3", "bulk"]
    for w in which:
        if w == "bulk":
            bulk()
        else:
            study(w, *{"c2": c2, "c3": c3}[w]())
