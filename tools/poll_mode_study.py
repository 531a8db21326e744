"""Poll-site flag pipelining vs synchronous flag test (CTXB_SYNC_POLL) on the
flag-mode configs: uninterrupted kernel time (poll cost) and preemption
latency (detection spread + routines) per mode.  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def setup(which):
    if which == "c4a":
        cfg = configs.c4a(1 << 28, grid=1)
        k = torch.from_numpy(cfg["buffers"]["keys"].view(np.int32)).cuda()
        st = torch.from_numpy(cfg["buffers"]["starts"].view(np.int32)).cuda()
        return cfg["ir"], lambda g: [k, st, torch.zeros(256 * g, dtype=torch.int32, device="cuda")], 0
    if which == "c3":
        cfg = configs.c3()
        x = torch.from_numpy(cfg["buffers"]["X"].view(np.int32)).cuda()
        return cfg["ir"], lambda g: [x, torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")], 0
    cfg = configs.c2()
    a = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    return cfg["ir"], lambda g: [a, b, torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")], 2


def main():
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    rows = ["| config | mode | regs | grid | kernel ms (median of 5) | routines µs p50 | flag-seen spread µs p50 | signal->drained µs p50 |",
            "|---|---|---|---|---|---|---|---|"]
    for which in sys.argv[1:] or ["c4a", "c3", "c2"]:
        txt, mk, mb = setup(which)
        base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=mb)
        bps, nsm = base.occupancy()
        for name, mode, fl in (("ctxback", 0, 0), ("ctxback sync", 0, cb.SYNC_POLL),
                               ("full_hw", 3, 0), ("full_hw sync", 3, cb.SYNC_POLL)):
            prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, mode=mode, flags=cb.ALL | fl, min_blocks_per_sm=bps)
            grid = min(bps, prog.occupancy()[0]) * nsm
            bufs = mk(grid)
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            ts = []
            for _ in range(5):
                run = prog.launch(grid, bufs, [], ctx, s)
                run.wait()
                ts.append(run.launch_ms())
                del run
            T = float(np.median(ts))
            lat, spread, s2d = [], [], []
            for fr in np.random.default_rng(3).uniform(0.1, 0.9, 7):
                run = prog.launch(grid, bufs, [], ctx, s)
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + fr * T / 1e3:
                    pass
                st = run.preempt(ctrl)
                if st["warps_preempted"]:
                    h = run.headers()
                    pre = (h[:, 2] == 1) & (h[:, 3] == 1)
                    stp = run.stamps()[pre].astype(np.int64)
                    lat.append(st["latency_us"])
                    spread.append((stp[:, 0].max() - stp[:, 0].min()) / 1e3)
                    s2d.append(st["signal_to_drained_us"])
                    run.resume(s)
                    run.wait()
                del run
            rows.append(f"| {which} | {name} | {prog.info['num_regs']} | {grid} | {T:.3f} | {np.median(lat):.2f} | "
                        f"{np.median(spread):.2f} | {np.median(s2d):.2f} |")
            print(rows[-1], flush=True)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
