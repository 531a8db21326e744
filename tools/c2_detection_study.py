"""C2 detection spread vs poll density: where do the ~3 us between the first
and the last warp seeing the flag come from?  Per variant (poll sites per
k-iteration, flag pipeline depth, synchronous test): uninterrupted kernel
time, routines span, flag-seen spread and its percentiles, per-warp save
time.  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402

VARIANTS = (("iter", 1, 0), ("iter", 1, cb.SYNC_POLL), ("iter", 2, 0), ("two", 1, 0), ("two", 1, cb.SYNC_POLL),
            ("step", 1, 0))


def main():
    trials = int(os.environ.get("TRIALS", "9"))
    modes = [(0, "ctxback"), (3, "full_hw")]
    cfg = configs.c2()
    a = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    c = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    rows = ["| polls | D | sync | mode | regs | kernel ms | routines µs p50 | spread µs p50 | seen-min p50/p90/p99 µs | "
            "save/warp µs p50 | signal->drained µs p50 |", "|---|---|---|---|---|---|---|---|---|---|---|"]
    for polls, depth, fl in VARIANTS:
        txt = configs.c2_ir(polls=polls)
        for mode, mname in modes:
            prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, mode=mode, flags=cb.ALL | fl,
                              min_blocks_per_sm=2, flag_depth=depth)
            bps, nsm = prog.occupancy()
            grid = bps * nsm
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            ts = []
            for _ in range(5):
                run = prog.launch(grid, [a, b, c], [], ctx, s)
                run.wait()
                ts.append(run.launch_ms())
                del run
            T = float(np.median(ts))
            lat, spread, sm, sw, s2d = [], [], [], [], []
            for fr in np.random.default_rng(3).uniform(0.1, 0.9, trials):
                run = prog.launch(grid, [a, b, c], [], ctx, s)
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + fr * T / 1e3:
                    pass
                st = run.preempt(ctrl)
                if st["warps_preempted"]:
                    h = run.headers()
                    pre = (h[:, 2] == 1) & (h[:, 3] == 1)
                    stp = run.stamps()[pre].astype(np.int64)
                    lat.append(st["latency_us"])
                    seen = (stp[:, 0] - stp[:, 0].min()) / 1e3
                    spread.append(seen.max())
                    sm.append(np.percentile(seen, [50, 90, 99]))
                    sw.append(np.median(stp[:, 1] - stp[:, 0]) / 1e3)
                    s2d.append(st["signal_to_drained_us"])
                    run.resume(s)
                    while not run.wait():
                        run.resume(s)
                del run
            q = np.median(np.array(sm), axis=0)
            rows.append(f"| {polls} | {depth} | {'y' if fl else 'n'} | {mname} | {prog.info['num_regs']} | {T:.3f} | "
                        f"{np.median(lat):.2f} | {np.median(spread):.2f} | {q[0]:.2f} / {q[1]:.2f} / {q[2]:.2f} | "
                        f"{np.median(sw):.2f} | {np.median(s2d):.2f} |")
            print(rows[-1], flush=True)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
