"""P:317 routine sharing: routines, cubin size and the uninterrupted kernel
time of C2 with 8 poll sites per k-iteration ("half") and C1-style programs,
for both sharing levels, exact sharing only, and no sharing.  GPU (kernel
times); prints a markdown table."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402


def main():
    cfg = configs.c2(polls="half")
    a = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    b = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    c = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    print("| program | sharing | routines | cubin bytes | kernel ms (polls) | no-polls ms | overhead |")
    print("|---|---|---|---|---|---|---|")
    for name, dbg in (("flashback-point + exact", 0), ("exact only", cb.DEBUG_NO_FP_SHARE), ("none", cb.DEBUG_NO_SHARE)):
        p = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, debug=dbg)
        info = p.info
        q = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, debug=dbg | cb.DEBUG_NO_POLLS)
        grid = p.persistent_grid()
        ts = {"p": [], "q": []}
        ctx = torch.empty(max(p.context_capacity(grid), q.context_capacity(grid)), dtype=torch.uint8, device="cuda")
        for i in range(8):
            for k, prog in (("p", p), ("q", q)):
                run = prog.launch(grid, [a, b, c], [], ctx)
                run.wait()
                if i:
                    ts[k].append(run.launch_ms())
                del run
        tp, tq = float(np.median(ts["p"])), float(np.median(ts["q"]))
        print(f"| C2, 8 sites / iteration | {name} | {info['n_save_stubs']} | {info['cubin_bytes']} | {tp:.3f} | "
              f"{tq:.3f} | {100 * (tp / tq - 1):.1f} % |", flush=True)


if __name__ == "__main__":
    main()
