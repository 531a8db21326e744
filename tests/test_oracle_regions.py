"""Pins of the idempotent-region heads h(c) (R-3) and of
CS-Defer's deferral targets, on hand-derived fixtures.

tests/golden/r3.json / r3bar.json: a kernel with an atomic, a load-then-store
(WAR) on one rw buffer followed by a second store to it, and a shared-memory
kernel with two barriers.  Every h(c) and the chosen flashback-point / bytes
at the sites after each cut are derived by hand (see the fixtures' `cite`);
the `no_cut_plans` show the plans a misreading of the cut would give, so the
cut is observable in the context bytes.  tests/golden/defer.json: the
deferral targets of CS-Defer and CTXBack+CS-Defer on r3's kernel, derived by
hand from the per-site context sizes.  The C++ analyzer is checked against
the same hand values (not only against the oracle).
"""
import json
import os

import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import ir

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    g = json.load(open(os.path.join(GOLD, name + ".json")))
    return g, ir.parse(g["ir"])


@pytest.mark.parametrize("name", ["r3", "r3bar"])
def test_region_heads_by_hand(name):
    g, op = load(name)
    assert A.region_heads(op) == g["heads"]


@pytest.mark.parametrize("name", ["r3", "r3bar"])
def test_plans_after_each_cut(name):
    g, op = load(name)
    s0 = op.bbs[op.labels["main"]][0]
    an = A.analyze(op)
    prog = cb.Program(g["ir"], debug=cb.DEBUG_NO_COMPILE)
    sites = list(an.sites)
    for k, (p, nbytes) in g["plans"].items():
        c = s0 + int(k)
        pl = an.plans[c]
        assert (pl.p - s0, pl.payload_bytes) == (p, nbytes), k
        si = prog.site_info(sites.index(c))
        assert (si["p"] - s0, si["payload_bytes_per_warp"]) == (p, nbytes), k


@pytest.mark.parametrize("name", ["r3", "r3bar"])
def test_misread_cut_changes_bytes(name):
    """The window without the cut (h = BB start) reaches the plan the fixture
    lists as `no_cut_plans`: the cut is what keeps the chosen plan."""
    g, op = load(name)
    s0 = op.bbs[op.labels["main"]][0]
    lv = A.liveness(op)
    bb_heads = [0] * len(op.instrs)
    for s, e in op.bbs:
        for c in range(s, e):
            bb_heads[c] = s
    for k, (p, nbytes) in g["no_cut_plans"].items():
        c = s0 + int(k)
        best = A.best_plan(op, lv, bb_heads, c, (), A.FLAGS_ALL)
        assert (best.p - s0, best.payload_bytes) == (p, nbytes)
        assert nbytes < g["plans"][k][1]


@pytest.mark.parametrize("mode", ["live", "ctxback"])
def test_defer_targets_by_hand(mode):
    d = json.load(open(os.path.join(GOLD, "defer.json")))
    g, op = load(d["ir_fixture"])
    s0 = op.bbs[op.labels["main"]][0]
    m = A.MODE_LIVE if mode == "live" else A.MODE_CTXBACK
    ib = d["defer_instr_bytes"]
    an = A.analyze(op, mode=m, flags=A.FLAGS_ALL | A.FLAG_DEFER, defer_instr_bytes=ib)
    main = [c for c in an.sites if c >= s0]
    assert [an.plans[c].payload_bytes for c in main] == d[f"{mode}_bytes_main"]
    assert [an.defer[c] - s0 for c in main] == d[f"targets_{mode}_main"]
    assert [an.defer[c] for c in an.sites if c < s0] == d["targets_init"]
    prog = cb.Program(g["ir"], flags=cb.ALL | cb.DEFER, mode=m, defer_instr_bytes=ib, debug=cb.DEBUG_NO_COMPILE)
    got = [prog.site_info(k)["defer_site"] for k in range(prog.num_sites)]
    want = d["targets_init"] + [t + len(d["targets_init"]) for t in d[f"targets_{mode}_main"]]
    assert got == want


def test_osrb_selection_by_hand():
    """R-7 on tests/golden/osrb_select.json: which irreversible
    scalar defs are candidates, which one is selected (the one whose backup
    lets a live result re-execute), and the plans with OSRB on / off at one
    site -- oracle and C++ analyzer against the hand values."""
    g, op = load("osrb_select")
    s0 = op.bbs[op.labels["main"]][0]
    assert [m - s0 for m in A.osrb_candidates(op)] == g["candidates"]
    an = A.analyze(op)
    assert [m - s0 for m in an.backups] == g["selected"]
    prog = cb.Program(g["ir"], debug=cb.DEBUG_NO_COMPILE)
    assert [m - s0 for m in prog.backups] == g["selected"]
    c = s0 + g["site"]
    assert (an.plans[c].p - s0, an.plans[c].payload_bytes) == tuple(g["osrb_on"])
    off = A.analyze(op, flags=A.FLAG_RELAXED | A.FLAG_REVERT)
    assert (off.plans[c].p - s0, off.plans[c].payload_bytes) == tuple(g["osrb_off"])
    poff = cb.Program(g["ir"], flags=cb.RELAXED | cb.REVERT, debug=cb.DEBUG_NO_COMPILE)
    k = an.sites.index(c)
    assert (poff.site_info(k)["p"] - s0, poff.site_info(k)["payload_bytes_per_warp"]) == tuple(g["osrb_off"])
    for lk, want in g["bytes_osrb_on_main"].items():
        cc = s0 + int(lk)
        assert an.plans[cc].payload_bytes == want
        assert prog.site_info(an.sites.index(cc))["payload_bytes_per_warp"] == want
