"""L2-cold in-situ resume against its cold-read floor: C2 and C3 (bench
placement), CTXBack and FULL_HW, flag at 50 % of T, 256 MiB written between
preempt and resume; the floor is ctxb_restore_floor of the payload plus the
replay's re-executed loads per warp on the same grid.  (The round-2 TMA L2
prefetch and speculative-prefix experiments that this study first compared
were not kept; profiles/r02_ncu_summary.md has their numbers.)
Usage: python tools/resume_floor_study.py [trials]"""
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


def setups():
    c2 = configs.c2()
    yield "c2", c2["ir"], [torch.from_numpy(c2["buffers"]["A"].view(np.int32)).cuda(),
                           torch.from_numpy(c2["buffers"]["B"].view(np.int32)).cuda(),
                           torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")], 2
    c3 = configs.c3(**configs.BENCH_C3)
    yield "c3", c3["ir"], [torch.from_numpy(c3["buffers"]["X"].view(np.int32)).cuda(),
                           torch.zeros(c3["W"] * c3["H"], dtype=torch.int32, device="cuda")], 0


def main():
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    print("| config | mode | resume µs p50 | floor µs (payload + replayed loads) | resume / floor |")
    print("|---|---|---|---|---|")
    for name, txt, bufs, mb in setups():
        for mode_name, mode in (("ctxback", 0), ("full_hw", 3)):
            prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, mode=mode, min_blocks_per_sm=mb)
            grid = prog.persistent_grid()
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            run = prog.launch(grid, bufs, [], ctx, s)
            run.wait()
            T = run.launch_ms() / 1e3
            del run
            res, byts = [], []
            for _ in range(trials):
                run = prog.launch(grid, bufs, [], ctx, s)
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + 0.5 * T:
                    pass
                run.preempt(ctrl)
                h = run.headers().copy()
                pre = (h[:, 2] == 1) & (h[:, 3] == 1)
                if pre.any():
                    with torch.cuda.stream(s):
                        scratch.fill_(1)
                    run.resume(s)
                    run.wait()
                    res.append(run.resume_stats()["resume_us"])
                    k = (h[pre, 0] & 0x7FFFFFFF).astype(np.int64)
                    rx = np.array([prog.site_info(int(x))["reexec_load_bytes_per_warp"] for x in k])
                    byts.append(float(np.max(h[pre, 1].astype(np.int64) + rx)))
                else:
                    run.wait()
                del run
            bpw = int(np.median(byts))
            fl = cb.ctxb_restore_floor(s, bpw, grid, 256, 9)
            r = float(np.median(res))
            print(f"| {name} | {mode_name} | {r:.2f} | {fl:.2f} ({bpw} B / warp) | {r / fl:.2f} |", flush=True)


if __name__ == "__main__":
    main()
