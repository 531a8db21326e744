"""Pins of the oracle's flashback analysis on the paper's worked examples.

Each fixture under tests/golden/ carries its PAPER.md citation.  Expected
register counts per candidate flashback-point and the chosen plans are the
paper's (Figs 2, 3, 4, 6) or, where the figure is lost (Fig 5) or the text is
silent (R-9), the SURVEY §8(c) hand derivation cited in the fixture.
"""
import json
import os

import numpy as np
import pytest

from oracle import analysis as A
from oracle import interp, ir

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    g = json.load(open(os.path.join(GOLD, name + ".json")))
    prog = ir.parse(g["ir"])
    s0 = prog.bbs[prog.labels["main"]][0]
    return g, prog, s0


def fmt_saved(pl, s0):
    out = []
    for src, (r, d) in pl.saved:
        out.append(f"{src}:{r}@{'PRE' if d is None else 'I%d' % (d - s0)}")
    return sorted(out)


def cands(prog, s0, site, flags=A.FLAGS_ALL, backups=()):
    lv = A.liveness(prog)
    c = s0 + site
    out = {}
    for p in range(s0, c + 1):
        out[p - s0] = A.plan_window(prog, lv, p, c, backups, flags)
    return out, lv, c


@pytest.mark.parametrize("name", ["fig2", "fig3", "fig4", "fig6"])
def test_figure_candidates_and_plan(name):
    g, prog, s0 = load(name)
    cs, lv, c = cands(prog, s0, g["site"])
    assert sorted(lv.live_in[c]) == g["live_in"]
    got = {str(p): (pl.payload_bytes // A.VEC_BYTES if pl else None) for p, pl in cs.items()}
    assert got == g["regs_per_p"]
    an = A.analyze(prog, sites=[c])
    pl = an.plans[c]
    assert pl.p - s0 == g["chosen_p"]
    assert fmt_saved(pl, s0) == sorted(g["saved"])
    assert sorted(j - s0 for j in pl.reexec_supply) == g["reexec"]
    assert sorted(e[1] - s0 for e in pl.preempt_reverts) == g["revert_pre"]
    res = sorted(pl.revert_info[e[1]][0] - s0 for e in pl.schedule if e[0] == "R")
    assert res == g["revert_res"]


def test_fig3_without_reverting():
    """without instruction reverting, I0 is not a flashback-point."""
    g, prog, s0 = load("fig3")
    cs, _lv, _c = cands(prog, s0, g["site"], flags=A.FLAG_RELAXED | A.FLAG_OSRB)
    got = {str(p): (pl.payload_bytes // A.VEC_BYTES if pl else None) for p, pl in cs.items()}
    assert got == g["norevert_regs_per_p"]


def test_fig4_value_ssa_two_values_of_r0():
    """Fig 4c: (r0, I2) is loaded, (r0, PRE) is computed by the revert and
    (r0, I2) is recomputed by re-executing I2 -- two values of r0 coexist."""
    g, prog, s0 = load("fig4")
    an = A.analyze(prog, sites=[s0 + g["site"]])
    pl = an.plans[s0 + g["site"]]
    sched = pl.schedule
    kinds = [(e[0], e[1] - s0 if e[0] == "X" else e[1]) for e in sched]
    # MUL #I0 first, then the revert of I2, then I1..I3 re-executed
    assert kinds[0] == ("X", 0)
    assert kinds[1][0] == "R" and kinds[1][1] == ("v0", None)
    assert [k for k in kinds[2:]] == [("X", 1), ("X", 2), ("X", 3)]


def test_fig5_osrb():
    g, prog, s0 = load("fig5")
    c = s0 + g["site"]
    lv = A.liveness(prog)
    assert sorted(lv.live_in[c]) == g["live_in"]
    off = {str(p - s0): A.plan_window(prog, lv, p, c, (), A.FLAG_RELAXED | A.FLAG_REVERT).payload_bytes
           for p in range(s0, c + 1)}
    assert off == g["bytes_per_p_osrb_off"]
    an_off = A.analyze(prog, sites=[c], flags=A.FLAG_RELAXED | A.FLAG_REVERT)
    assert an_off.plans[c].p - s0 == g["chosen_p_osrb_off"]
    an = A.analyze(prog, sites=[c])
    assert an.backups == [s0 + 1]              # the scalar load I1 is backed up
    on = {str(p - s0): A.plan_window(prog, lv, p, c, an.backups).payload_bytes for p in range(s0, c + 1)}
    assert on == g["bytes_per_p_osrb_on"]
    assert an.plans[c].p - s0 == g["chosen_p_osrb_on"]
    assert fmt_saved(an.plans[c], s0) == sorted(g["saved_osrb_on"])


def test_r9_per_p_recomputation():
    g, prog, s0 = load("r9")
    cs, _lv, c = cands(prog, s0, g["site"])
    got = {str(p): (pl.payload_bytes // A.VEC_BYTES if pl else None) for p, pl in cs.items()}
    assert got == g["regs_per_p"]
    for p, sv in g["saved_at_p"].items():
        assert fmt_saved(cs[int(p)], s0) == sorted(sv)
    an = A.analyze(prog, sites=[c])
    assert an.plans[c].p - s0 == g["chosen_p"]


@pytest.mark.parametrize("name", ["fig2", "fig3", "fig4", "fig5", "fig6", "r9"])
def test_every_candidate_plan_replays(name):
    """BF1 on the worked examples: for every site and every feasible
    flashback-point, preempting there, poisoning every register and
    replaying the plan gives the uninterrupted result."""
    g, prog, s0 = load(name)
    an = A.analyze(prog)
    rng = np.random.default_rng(5)
    bufs = {}
    for b, kind in prog.buffers.items():
        bufs[b] = rng.integers(0, 64, 64, dtype=np.uint32) if kind == "ro" else np.zeros(64, np.uint32)
    ref, _ = interp.run(an, 1, bufs)
    lv = an.lv
    for c in an.sites:
        for p in range(an.heads[c], c + 1):
            pl = A.plan_window(prog, lv, p, c, an.backups)
            if pl is None:
                continue
            forced = A.Analysis(prog, lv, an.sites, an.heads, an.backups, dict(an.plans), an.live)
            forced.plans[c] = pl
            k = an.sites.index(c)
            out, rec = interp.run(forced, 1, bufs, schedule=[[k]])
            assert rec and rec[0]["site"] == c and rec[0]["bytes"] == pl.payload_bytes
            for b in ref:
                assert np.array_equal(out[b], ref[b]), (name, c, p, b)
