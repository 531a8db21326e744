"""One polled flag word vs CTXB_FLAG_REPLICAS (master pollers + 64 replicas)
per config: uninterrupted kernel time, the same kernel with polls compiled out,
preemption routines and signal -> drained (flag mode, 9 trials).  GPU; prints
a markdown table."""
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
        return cfg["ir"], lambda g: [k, st, torch.zeros(256 * g, dtype=torch.int32, device="cuda")], 0, cb.SYNC_POLL
    if which.startswith("c3"):
        cfg = configs.c3(rows_per_iter=int(which[3:]) if which.startswith("c3r") else 1)
        x = torch.from_numpy(cfg["buffers"]["X"].view(np.int32)).cuda()
        return cfg["ir"], lambda g: [x, torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")], 0, 0
    cfg = configs.c2() if which == "c2" else configs.c2s()
    a = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    return cfg["ir"], lambda g: [a, b, torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")], 2, 0


def kernel_ms(prog, grid, bufs, ctx, s, n=7):
    ts = []
    for _ in range(n):
        run = prog.launch(grid, bufs, [], ctx, s)
        run.wait()
        ts.append(run.launch_ms())
        del run
    return float(np.median(ts))


def main():
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    rows = ["| config | flag | kernel ms | no-polls ms | overhead | routines µs p50 | signal->drained µs p50 |",
            "|---|---|---|---|---|---|---|"]
    for which in sys.argv[1:] or ["c2", "c2s", "c3", "c4a"]:
        txt, mk, mb, extra = setup(which)
        base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=mb, flags=cb.ALL | extra,
                          debug=cb.DEBUG_NO_POLLS)
        bps, nsm = base.occupancy()
        grid = bps * nsm
        bufs = mk(grid)
        ctx = torch.empty(base.context_capacity(grid), dtype=torch.uint8, device="cuda")
        t0_ms = kernel_ms(base, grid, bufs, ctx, s)
        variants = [(f"{nm}, load every {k}", fl, k) for k in [int(x) for x in os.environ.get("LOADS", "1").split(",")]
                    for nm, fl in (("one word", 0), ("replicas", cb.FLAG_REPLICAS))]
        for name, fl, k in variants:
            prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=mb, flags=cb.ALL | extra | fl,
                              load_every=k)
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            T = kernel_ms(prog, grid, bufs, ctx, s)
            lat, s2d = [], []
            for fr in np.random.default_rng(3).uniform(0.1, 0.9, 9):
                run = prog.launch(grid, bufs, [], ctx, s)
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + fr * T / 1e3:
                    pass
                st = run.preempt(ctrl)
                if st["warps_preempted"]:
                    lat.append(st["latency_us"])
                    s2d.append(st["signal_to_drained_us"])
                    run.resume(s)
                    while not run.wait():
                        run.resume(s)
                del run
            rows.append(f"| {which} | {name} | {T:.3f} | {t0_ms:.3f} | {100 * (T / t0_ms - 1):.1f} % | "
                        f"{np.median(lat):.2f} | {np.median(s2d):.2f} |")
            print(rows[-1], flush=True)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
