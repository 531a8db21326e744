"""Restore efficiency for small, L2-cold contexts (C2's in-situ restore is
21 MB): bulk restore through the generated stubs vs plain torch read-only
kernels over the same bytes, each after a 256 MiB L2 eviction.  Kernel
durations from CUDA events; prints a markdown table."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def main():
    s = torch.cuda.Stream()
    scratch = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
    prog = cb.Program(configs.bulk_ir(64), poll_policy=cb.POLL_EXPLICIT, mode=cb.MODE_LIVE, debug=cb.DEBUG_FORCED)
    rows = ["| MiB | warps | stub restore µs (cold) | GB/s | stub save µs | torch sum µs (cold) | GB/s | "
            "torch sum µs (warm) |", "|---|---|---|---|---|---|---|---|"]
    for mib in (8, 21, 40, 84, 256):
        nw = (mib << 20) // 8192
        grid = nw // 8
        nw = grid * 8
        out = torch.zeros(256, dtype=torch.int32, device="cuda")
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        zeros, never = np.zeros(nw, np.uint32), np.full(nw, cb.NEVER, np.uint32)
        rest, save = [], []
        for i in range(7):
            run = prog.launch(grid, [out], [], ctx, s, forced=zeros)
            assert not run.wait()
            save.append(run.launch_ms())
            with torch.cuda.stream(s):
                scratch.fill_(i)
            run.resume(s, forced=never)
            assert run.wait()
            rest.append(run.launch_ms())
            del run
        x = torch.ones(nw * 2048, dtype=torch.float32, device="cuda")
        cold, warm = [], []
        for i in range(7):
            with torch.cuda.stream(s):
                scratch.fill_(i)
                e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                e0.record(s)
                x.sum()
                e1.record(s)
                x.sum()
                e2.record(s)
            s.synchronize()
            cold.append(e0.elapsed_time(e1))
            warm.append(e1.elapsed_time(e2))
        b = nw * 8192
        r, c = np.median(rest[2:]) * 1e3, np.median(cold[2:]) * 1e3
        rows.append(f"| {mib} | {nw} | {r:.2f} | {b / r / 1e3:.0f} | {np.median(save[2:]) * 1e3:.2f} | {c:.2f} | "
                    f"{b / c / 1e3:.0f} | {np.median(warm[2:]) * 1e3:.2f} |")
        print(rows[-1], flush=True)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
