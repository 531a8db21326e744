"""Static context-size study (the analogue of the paper's Fig. 7):
every instruction of each config kernel is a preemption point; per point the
context of BASELINE (FULL_HW: all registers the compiled kernel occupies),
FULL_IR, LIVE and CTXBack, and the "minimum possible context" analogue
min_{p in window} LIVE_IN(p) (R-13; the paper's CKPT bound).  Averages
are of per-kernel normalised values, as in the paper.

CPU only: plans from libctxb's analyzer (NO_COMPILE), liveness / windows from
the oracle, register counts from NVRTC.  Writes profiles/r01_context_stats.md."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402
from oracle import analysis as A  # noqa: E402
from oracle import ir  # noqa: E402
from workloads import configs  # noqa: E402

KERNELS = [
    ("C1 k24", configs.c1()["ir"], 0),
    ("C2 sgemm 128x128x16", configs.c2_ir(128, 128, 16), 2),
    ("C3 stencil", configs.c3_ir(512, 128, 64), 0),
    ("C4a histogram", configs.c4a_ir(1 << 14), 0),
    ("C4b bfs", configs.c4b_ir(), 0),
]


def study(name, txt, minb):
    op = ir.parse(txt)
    lv = A.liveness(op)
    heads = A.region_heads(op)
    full_ir = A.full_ir_bytes(op)
    prog = cb.Program(txt, poll_policy=cb.POLL_EVERY_INSTR, debug=cb.DEBUG_NO_COMPILE)
    pol = cb.POLL_EXPLICIT if "poll" in txt else cb.POLL_EVERY_INSTR   # the kernel as benchmarked
    hw = cb.Program(txt, poll_policy=pol, mode=cb.MODE_FULL_HW, min_blocks_per_sm=minb)
    regs = hw.info["num_regs"]
    full_hw = max(regs * 128, full_ir)
    live_bytes = [sum(128 if r[0] == "v" else 4 for r in lv.live_in[i]) for i in range(len(op.instrs))]
    rows = []
    for k in range(prog.num_sites):
        si = prog.site_info(k)
        c = si["c"]
        mn = min(live_bytes[p] for p in range(heads[c], c + 1))
        rows.append((si["payload_bytes_per_warp"], si["live_bytes_per_warp"], mn, si["c"] - si["p"],
                     si["n_revert_pre"] + si["n_revert_res"]))
    a = np.array(rows, dtype=np.float64)
    ctx, live, mn, back, rev = a.T
    return dict(name=name, instrs=len(op.instrs), regs=regs, full_hw=full_hw, full_ir=full_ir,
                ctx_vs_hw=float(np.mean(ctx / full_hw)), live_vs_hw=float(np.mean(live / full_hw)),
                ctx_vs_live=float(np.mean(ctx[live > 0] / live[live > 0])) if (live > 0).any() else 1.0,
                ctx_vs_min=float(np.mean(ctx[mn > 0] / mn[mn > 0])) if (mn > 0).any() else float("nan"),
                at_min=float(np.mean(ctx <= mn)),
                mean_back=float(np.mean(back)), frac_revert=float(np.mean(rev > 0)),
                backups=len(prog.backups))


def main():
    res = [study(*k) for k in KERNELS]
    lines = ["# Round 1 — static context study (every instruction a preemption point)", "",
             "Analogue of the paper's Fig. 7 (P:339-347).  BASELINE = FULL_HW (every register the compiled",
             "kernel occupies x 128 B per warp, ptxas count), LIVE = LIVE_IN(I_cur) (P:337), CTXBack = the",
             "chosen plan's saved values (R-8).  Reduction = 1 - mean(context / FULL_HW) per kernel.",
             "'x min' = mean over points of CTXBack / min_{p in window} LIVE_IN(p) (R-13, the paper's 1.09x",
             "analogue; points whose window minimum is 0 B -- e.g. at kernel entry -- excluded); 'at/below min' = share of",
             "points where CTXBack's context is <= that minimum (it can be lower: CTXBack may save results instead",
             "of inputs, so min LIVE_IN(p) is not a lower bound for it).", "",
             "| kernel | instrs | regs | FULL_HW B/warp | LIVE reduction | CTXBack reduction | CTXBack / LIVE | CTXBack x min | at/below min | mean flashback distance | sites using a revert | OSRB backups |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in res:
        lines.append(f"| {r['name']} | {r['instrs']} | {r['regs']} | {r['full_hw']} | {100 * (1 - r['live_vs_hw']):.1f} % "
                     f"| {100 * (1 - r['ctx_vs_hw']):.1f} % | {r['ctx_vs_live']:.3f} | " + (f"{r['ctx_vs_min']:.3f}" if r['ctx_vs_min'] == r['ctx_vs_min'] else '— (window min 0 B)') + " "
                     f"| {100 * r['at_min']:.1f} % "
                     f"| {r['mean_back']:.1f} | {100 * r['frac_revert']:.1f} % | {r['backups']} |")
    lv = np.mean([1 - r["live_vs_hw"] for r in res])
    cx = np.mean([1 - r["ctx_vs_hw"] for r in res])
    mn = np.nanmean([r["ctx_vs_min"] for r in res])
    lines += ["", f"Average over the five kernels: LIVE reduces the context by {100 * lv:.1f} %, CTXBack by "
              f"{100 * cx:.1f} %, CTXBack context = {mn:.3f} x the window-minimum LIVE context.",
              "Paper (AMD Radeon VII, 12 OpenCL kernels, context only): LIVE 37.8 %, CTXBack 61.0 %, 1.09 x of "
              "the minimum (P:345)."]
    out = "\n".join(lines) + "\n"
    print(out)
    path = os.path.join(ROOT, "profiles", "r01_context_stats.md")
    open(path, "w").write(out)


if __name__ == "__main__":
    main()
