"""Poll-site overhead of the synchronous flag test (CTXB_SYNC_POLL) next to
the pipelined default, with the drain notice's exit counting in both builds,
on each config's bench placement (polled vs no-polls build, interleaved, each
kernel's own persistent grid).  GPU; prints a markdown table."""
import os
import sys

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
    c3 = configs.c3(**configs.BENCH_C3)
    x = torch.from_numpy(c3["buffers"]["X"].view(np.int32)).cuda()
    y = torch.zeros(c3["W"] * c3["H"], dtype=torch.int32, device="cuda")
    c4 = configs.c4a(1 << 28, grid=1)
    k = torch.from_numpy(c4["buffers"]["keys"].view(np.int32)).cuda()
    st = torch.from_numpy(c4["buffers"]["starts"].view(np.int32)).cuda()
    h = torch.zeros(256 * 4096, dtype=torch.int32, device="cuda")
    cases = [("c2", c2["ir"], lambda: [a, b, c], 2, 0), ("c2s", configs.c2s()["ir"], lambda: [a, b, c], 2, 0),
             ("c3", c3["ir"], lambda: [x, y], 0, 0), ("c4a", c4["ir"], lambda: [k, st, h.zero_()], 0, 0)]
    if os.environ.get("C4A_MID"):       # only C4a, with extra sites inside the atomics
        cases = [(f"c4a_m{m}", configs.c4a_ir(1 << 28, 8, m), lambda: [k, st, h.zero_()], 0, 0)
                 for m in (0, 1, 3)]
    if os.environ.get("C4A_PL"):        # only C4a, with other chunk sizes (keys per lane)
        cases = []
        for p in os.environ["C4A_PL"].split(","):
            cp = configs.c4a(1 << 28, grid=1, per_lane=int(p))      # its own chunk starts
            stp = torch.from_numpy(cp["buffers"]["starts"].view(np.int32)).cuda()
            cases.append((f"c4a_p{p}", cp["ir"], lambda stp=stp: [k, stp, h.zero_()], 0, 0))
    print("| config | flag test | polled ms | no-polls ms | overhead |")
    print("|---|---|---|---|---|")
    for name, txt, mk, mb, ex in cases:
        for tname, fl in (("pipelined", 0), ("sync", cb.SYNC_POLL)):
            r = bench._poll_overhead(cb, txt, None, mk, extra_flags=ex | fl | cb.DRAIN_NOTICE, min_blocks=mb)
            print(f"| {name} | {tname} | {r['polls_ms']:.3f} | {r['no_polls_ms']:.3f} | {r['overhead_pct']:.1f} % |",
                  flush=True)


if __name__ == "__main__":
    main()
