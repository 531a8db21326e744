"""CTXB_WATCHER study: the preemption signal through the stream memory op,
the armed (pre-enqueued) memop, and the co-resident watcher warp that relays
a host store (with and without the memop fallback).  Per config and mode:
uninterrupted kernel time on the persistent grid (ctxb_persistent_grid: one
block fewer on C2, whose SMs have no room for the watcher otherwise),
host-clock preemption latency (ctxb_preempt entry -> victim stream drained),
the device-side routines span and the flag-seen spread; outputs checked
against the uninterrupted run.  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def setup(which):
    if which.startswith("c4a"):          # c4a, c4a_m1, c4a_m3: extra poll sites inside the atomics; c4a_p4: 4 keys / lane
        cfg = configs.c4a(1 << 28, grid=1, mid_polls=int(which[5:]) if "_m" in which else 0,
                          per_lane=int(which[5:]) if "_p" in which else 8)
        k = torch.from_numpy(cfg["buffers"]["keys"].view(np.int32)).cuda()
        st = torch.from_numpy(cfg["buffers"]["starts"].view(np.int32)).cuda()
        return cfg["ir"], lambda g: [k, st, torch.zeros(256 * g, dtype=torch.int32, device="cuda")], 0, cb.SYNC_POLL
    if which == "c3":
        cfg = configs.c3(**configs.BENCH_C3)
        x = torch.from_numpy(cfg["buffers"]["X"].view(np.int32)).cuda()
        return cfg["ir"], lambda g: [x, torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")], 0, 0
    cfg = configs.c2()
    a = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    return cfg["ir"], lambda g: [a, b, torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")], 2, 0


MODES = (("memop", 0, None, None), ("armed", cb.ARMED_SIGNAL, None, None),
         ("watcher", cb.WATCHER, None, None), ("watcher only", cb.WATCHER, None, "1"),
         ("watcher + drain notice", cb.WATCHER | cb.DRAIN_NOTICE, None, None),
         ("armed + drain notice", cb.ARMED_SIGNAL | cb.DRAIN_NOTICE, None, None))
if os.environ.get("MODES") == "headline":    # the bench's signal path only
    MODES = (("watcher + drain notice + sync poll", cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL, None, None),)
if os.environ.get("MODES") == "sync":      # the synchronous flag test on the headline path
    MODES = (("watcher + drain notice", cb.WATCHER | cb.DRAIN_NOTICE, None, None),
             ("watcher + drain notice + sync poll", cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL, None, None))


def main():
    trials = int(os.environ.get("TRIALS", "15"))
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    rows = ["| config | signal | grid | kernel ms (median of 5) | host latency µs p50 / p90 | signal->drained µs p50 (events) | "
            "routines µs p50 | flag-seen spread µs p50 | preempted |",
            "|---|---|---|---|---|---|---|---|---|"]
    # host latency: ctxb_preempt entry -> victim drained (host clock); events: signal event -> drained
    for which in sys.argv[1:] or ["c2", "c3", "c4a"]:
        txt, mk, mb, extra = setup(which)
        for name, fl, relays, only in MODES:
            os.environ.pop("CTXB_HOST_RELAYS", None)
            os.environ.pop("CTXB_HOST_SIGNAL_ONLY", None)
            if relays:
                os.environ["CTXB_HOST_RELAYS"] = relays
            if only:
                os.environ["CTXB_HOST_SIGNAL_ONLY"] = only
            prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | fl | extra, min_blocks_per_sm=mb)
            grid = prog.persistent_grid()
            bufs = mk(grid)
            ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
            ts = []
            for _ in range(5):
                if which.startswith("c4a"):
                    bufs[-1].zero_()
                run = prog.launch(grid, bufs, [], ctx, s)
                run.wait()
                ts.append(run.launch_ms())
                del run
            T = float(np.median(ts))
            ref = bufs[-1].clone()
            host, lat, spread, s2d, npre = [], [], [], [], 0
            for fr in np.random.default_rng(3).uniform(0.1, 0.9, trials):
                if which.startswith("c4a"):
                    bufs[-1].zero_()
                run = prog.launch(grid, bufs, [], ctx, s)
                t0 = time.perf_counter()
                while time.perf_counter() < t0 + fr * T / 1e3:
                    pass
                st = run.preempt(ctrl)
                if st["warps_preempted"]:
                    npre += 1
                    h = run.headers()
                    pre = (h[:, 2] == 1) & (h[:, 3] == 1)
                    stp = run.stamps()[pre].astype(np.int64)
                    host.append(st["host_us"])
                    lat.append(st["latency_us"])
                    spread.append((stp[:, 0].max() - stp[:, 0].min()) / 1e3)
                    s2d.append(st["signal_to_drained_us"])
                    run.resume(s)
                    while not run.wait():
                        run.resume(s)
                else:
                    run.wait()
                torch.cuda.synchronize()
                assert torch.equal(bufs[-1], ref), f"{which} {name}: output differs"
                del run
            torch.cuda.synchronize()
            rows.append(f"| {which} | {name} | {grid} | {T:.3f} | {np.median(host):.2f} / {np.percentile(host, 90):.2f} | "
                        f"{np.median(s2d):.2f} | {np.median(lat):.2f} | {np.median(spread):.2f} | {npre}/{trials} |")
            print(rows[-1], flush=True)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
