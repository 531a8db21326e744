"""Speculative restore loads: L2-cold in-situ resume of C2 and
C3 (bench placement), CTXBack and FULL_HW, with the register budget of the
payload loads issued together with the header (`CTXB_SPEC_RESTORE_REGS`, read
when a program is generated; 0 = the payload loads wait for the header's
dispatch).  Flag at 50 % of T, 256 MiB written between preempt and resume,
runs of all budgets interleaved trial by trial.
Usage: python tools/spec_restore_study.py [trials] [budgets, e.g. 0,16,32,128]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

trials = int(sys.argv[1]) if len(sys.argv) > 1 else 9
budgets = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "0,16,32,128").split(",")]
scratch = torch.empty(64 << 20, dtype=torch.int32, device="cuda")


def setups():
    c2 = configs.c2()
    yield "c2", c2["ir"], [torch.from_numpy(c2["buffers"]["A"].view(np.int32)).cuda(),
                           torch.from_numpy(c2["buffers"]["B"].view(np.int32)).cuda(),
                           torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")], 2
    c3 = configs.c3(**configs.BENCH_C3)
    yield "c3", c3["ir"], [torch.from_numpy(c3["buffers"]["X"].view(np.int32)).cuda(),
                           torch.zeros(c3["W"] * c3["H"], dtype=torch.int32, device="cuda")], 0


def one(prog, grid, bufs, ctx, s, ctrl, T):
    run = prog.launch(grid, bufs, [], ctx, s)
    t0 = time.perf_counter()
    while time.perf_counter() < t0 + 0.5 * T:
        pass
    st = run.preempt(ctrl)
    r = None
    if st["warps_preempted"]:
        with torch.cuda.stream(s):
            scratch.fill_(1)
        run.resume(s)
        run.wait()
        r = run.resume_stats()["resume_us"]
    else:
        run.wait()
    del run
    return r


def main():
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    print("| config | mode | budget (regs) | speculated loads | regs resume | spill B | resume µs p50 | p10-p90 |")
    print("|---|---|---|---|---|---|---|---|")
    for name, txt, bufs, mb in setups():
        for mode_name, mode in (("ctxback", 0), ("full_hw", 3)):
            progs = {}
            for b in budgets:
                os.environ["CTXB_SPEC_RESTORE_REGS"] = str(b)
                progs[b] = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, mode=mode, min_blocks_per_sm=mb)
            os.environ.pop("CTXB_SPEC_RESTORE_REGS", None)
            grid = min(p.persistent_grid() for p in progs.values())
            ctxs = {b: torch.empty(p.context_capacity(grid), dtype=torch.uint8, device="cuda")
                    for b, p in progs.items()}
            run = progs[budgets[0]].launch(grid, bufs, [], ctxs[budgets[0]], s)
            run.wait()
            T = run.launch_ms() / 1e3
            del run
            res = {b: [] for b in budgets}
            for b in budgets:   # warm-up
                one(progs[b], grid, bufs, ctxs[b], s, ctrl, T)
            for _ in range(trials):
                for b in budgets:
                    r = one(progs[b], grid, bufs, ctxs[b], s, ctrl, T)
                    if r is not None:
                        res[b].append(r)
            for b in budgets:
                p = progs[b]
                nspec = p.source.count("_spec(pay")
                x = np.array(res[b])
                print(f"| {name} | {mode_name} | {b} | {nspec} | {p.info['num_regs_resume']} | "
                      f"{p.info['spill_stores_resume']} | {np.median(x):.2f} | "
                      f"{np.percentile(x, 10):.2f}-{np.percentile(x, 90):.2f} |", flush=True)


if __name__ == "__main__":
    main()
