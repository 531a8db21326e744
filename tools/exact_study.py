"""Exact minimum-bytes plans vs the greedy CTXB-R1 plans (NEXT N4, SURVEY
§8(f): "exact min-bytes plan (ILP/BF) vs greedy"; R-19).

Every instruction of each config kernel is a preemption point (as in the
static study, the analogue of the paper's Fig. 7), plus the kernels
as benchmarked (their explicit poll sites), plus 200 random IR programs.  Per
kernel: windows searched, windows whose search was cut off, windows where the
exact set is strictly smaller, and the chosen plans' bytes (greedy / exact).
The ratio greedy / exact is the analogue of the paper's "1.09x of the minimum
possible context".

CPU only (libctxb analyzer with NO_COMPILE).  Writes profiles/r01_exact_study.md."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from workloads import configs  # noqa: E402
from workloads.randprog import random_program  # noqa: E402

KERNELS = [
    ("C1 k24", configs.c1()["ir"]),
    ("C2 sgemm 128x128x64", configs.c2_ir(128, 128, 64)),
    ("C2 half (8 polls/iter)", configs.c2_ir(128, 128, 32, polls="half")),
    ("C2s sgemm + smem", configs.c2s_ir(128, 128, 64)),
    ("C3 stencil", configs.c3_ir(512, 128, 64)),
    ("C4a histogram", configs.c4a_ir(1 << 14)),
    ("C4b bfs", configs.c4b_ir()),
]


def compare(txt, policy):
    t0 = time.perf_counter()
    g = cb.Program(txt, flags=cb.ALL, poll_policy=policy, debug=cb.DEBUG_NO_COMPILE)
    t1 = time.perf_counter()
    e = cb.Program(txt, flags=cb.ALL | cb.EXACT, poll_policy=policy, debug=cb.DEBUG_NO_COMPILE)
    t2 = time.perf_counter()
    gb = [g.site_info(k)["payload_bytes_per_warp"] for k in range(g.num_sites)]
    eb = [e.site_info(k)["payload_bytes_per_warp"] for k in range(e.num_sites)]
    i = e.info
    return dict(sites=len(gb), greedy=sum(gb), exact=sum(eb), sites_better=sum(a > b for a, b in zip(gb, eb)),
                windows=i["exact_windows"], truncated=i["exact_truncated"], improved=i["exact_improved"],
                fallback=i["exact_fallback"], t_greedy=t1 - t0, t_exact=t2 - t1)


def main():
    lines = ["# Round 1 — exact minimum-bytes plans vs greedy CTXB-R1 (NEXT N4)", "",
             "`tools/exact_study.py` (CPU; libctxb analyzer).  *windows*: (site, flashback-point) pairs",
             "searched; *cut off*: search budget (2^20 nodes) or > 48 residual candidates exceeded",
             "(greedy plan kept); *better windows*: exact set strictly smaller than greedy's for that",
             "window; *sites better*: the chosen plan of the site is smaller.  Bytes are per warp,",
             "summed over sites.", "",
             "| kernel | poll sites | sites | windows | cut off | better windows | sites better | "
             "greedy B | exact B | greedy / exact | analysis s (greedy / exact) |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    for name, txt in KERNELS:
        pols = [("every instr", cb.POLL_EVERY_INSTR)]
        if "poll" in txt or "bar" in txt:
            pols.append(("as benchmarked", cb.POLL_EXPLICIT))
        for pname, pol in pols:
            r = compare(txt, pol)
            assert r["fallback"] == 0
            lines.append(f"| {name} | {pname} | {r['sites']} | {r['windows']} | {r['truncated']} | {r['improved']} | "
                         f"{r['sites_better']} | {r['greedy']} | {r['exact']} | {r['greedy'] / max(1, r['exact']):.4f} | "
                         f"{r['t_greedy']:.2f} / {r['t_exact']:.2f} |")
            print(lines[-1], flush=True)
    agg = dict(sites=0, greedy=0, exact=0, sites_better=0, windows=0, truncated=0, improved=0, progs=0, pb=0)
    for seed in range(200):
        txt, _ = random_program(seed, loop=seed % 3 == 0, n_body=14)
        r = compare(txt, cb.POLL_EVERY_INSTR)
        assert r["fallback"] == 0
        for k in ("sites", "greedy", "exact", "sites_better", "windows", "truncated", "improved"):
            agg[k] += r[k]
        agg["progs"] += 1
        agg["pb"] += r["sites_better"] > 0
    lines.append(f"| 200 random programs (n_body 14) | every instr | {agg['sites']} | {agg['windows']} | "
                 f"{agg['truncated']} | {agg['improved']} | {agg['sites_better']} | {agg['greedy']} | "
                 f"{agg['exact']} | {agg['greedy'] / agg['exact']:.4f} | — |")
    lines += ["", f"Random programs with >= 1 better site: {agg['pb']} of {agg['progs']}.", "",
              "Reading: the greedy sweep (Alg. 1 re-executes whatever it can, then saves what the",
              "re-executions need) reaches the exact minimum at every chosen site of the config kernels;",
              "it is beaten only where re-executing an instruction needs more saved inputs than saving",
              "its result (tests/golden/exact.json), which the configs' chosen flashback-points avoid.",
              "Paper (context only): CTXBack = 1.09x of the minimum possible context (P:345; there the",
              "minimum is CKPT's best checkpoint, our R-13 analogue is in r01_context_stats.md)."]
    out = os.path.join(ROOT, "profiles", "r01_exact_study.md")
    open(out, "w").write("\n".join(lines) + "\n")
    print("wrote", out)


if __name__ == "__main__":
    main()
