"""C2 poll density on the bench's signal path (watcher + drain notice +
synchronous test): one site per k-iteration ("iter", the bench) vs two
("two"): uninterrupted kernel time, poll overhead against the no-polls
build, host-observed preemption latency and routines span (25 flag
preemptions).  GPU; prints a markdown table."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def main():
    c2 = configs.c2()
    a = torch.from_numpy(c2["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(c2["buffers"]["B"].view(np.int32)).cuda()
    c = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    s = torch.cuda.Stream()
    fl = cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL
    bench.SIGNAL_FLAGS = fl
    print("| polls | kernel ms | overhead | host latency p50 / p90 | routines p50 | context / TB |")
    print("|---|---|---|---|---|---|")
    for polls in ("iter", "two"):
        txt = configs.c2_ir(polls=polls)
        ov = bench._poll_overhead(cb, txt, None, lambda: [a, b, c], min_blocks=2)
        prog = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, flags=cb.ALL | fl)
        grid = prog.persistent_grid()
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        run = prog.launch(grid, [a, b, c], [], ctx, s)
        run.wait()
        T = run.launch_ms() / 1e3
        del run
        host, lat, byt = [], [], []
        for fr in np.random.default_rng(3).uniform(0.1, 0.9, 25):
            run = prog.launch(grid, [a, b, c], [], ctx, s)
            t0 = time.perf_counter()
            while time.perf_counter() < t0 + fr * T:
                pass
            st = run.preempt(None)
            if st["warps_preempted"]:
                host.append(st["host_us"])
                lat.append(st["latency_us"])
                byt.append(st["payload_bytes"] / max(1, st["blocks_preempted"]))
                run.resume(s)
            run.wait()
            del run
        print(f"| {polls} | {T * 1e3:.3f} | {ov['overhead_pct']:.1f} % | {np.median(host):.2f} / "
              f"{np.percentile(host, 90):.2f} µs | {np.median(lat):.2f} µs | {np.median(byt):.0f} B |", flush=True)


if __name__ == "__main__":
    main()
