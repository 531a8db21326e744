"""Exact minimum-bytes plans (CTXB_EXACT, NEXT N4 "exact min-bytes plan vs
greedy", R-19) — oracle pins and C++ parity (no GPU).

Pins of oracle/exact.py against things other than itself:
* the paper's worked examples: the exact minimum per candidate flashback-point
  equals the figures' context sizes (Figs 2, 3, 4, 6);
* two hand-derived programs where the greedy CTXB-R1 sweep (Alg. 1 re-executes
  whatever it can) saves more than the minimum (tests/golden/exact.json);
* the independent greedy sweep: exact <= greedy for every window;
* oracle/brute.py's BF2 (a separate coding of the closure): exact == BF-min;
* replays: poisoned preempt/resume through the interpreter equals the
  uninterrupted run for every exact plan.
C++ parity: plan text of every site equals the oracle's.
"""
import json
import os

import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import brute, interp, ir
from oracle.exact import ExactWindow
from workloads import configs
from workloads.randprog import random_buffers, random_program

GOLD = os.path.join(os.path.dirname(__file__), "golden")
EXACT = A.FLAGS_ALL | A.FLAG_EXACT


def _fmt(pl, s0):
    return [f"{src}:{r}@{'PRE' if d is None else 'I%d' % (d - s0)}" for src, (r, d) in pl.saved]


@pytest.mark.parametrize("name", ["fig2", "fig3", "fig4", "fig6"])
def test_exact_matches_paper_figures(name):
    g = json.load(open(os.path.join(GOLD, name + ".json")))
    op = ir.parse(g["ir"])
    s0 = op.bbs[op.labels["main"]][0]
    c = s0 + g["site"]
    lv = A.liveness(op)
    got = {str(p - s0): ExactWindow(op, lv, p, c, (), A.FLAGS_ALL).plan().payload_bytes // A.VEC_BYTES
           for p in range(s0, c + 1)}
    assert got == g["regs_per_p"]
    an = A.analyze(op, sites=[c], flags=EXACT)
    assert an.plans[c].p - s0 == g["chosen_p"]
    assert sorted(_fmt(an.plans[c], s0)) == sorted(g["saved"])


@pytest.mark.parametrize("k", [0, 1])
def test_exact_hand_derived_cases(k):
    case = json.load(open(os.path.join(GOLD, "exact.json")))["cases"][k]
    op = ir.parse(case["ir"])
    s0 = op.bbs[op.labels["main"]][0]
    c = s0 + case["site"]
    lv = A.liveness(op)
    assert sorted(lv.live_in[c]) == case["live_in"]
    ex, gr = {}, {}
    for p in range(s0, c + 1):
        ex[str(p - s0)] = ExactWindow(op, lv, p, c, (), A.FLAGS_ALL).plan().payload_bytes
        g = A.plan_window(op, lv, p, c, (), A.FLAGS_ALL)
        gr[str(p - s0)] = g.payload_bytes if g else None
    assert ex == case["exact_bytes_per_p"]
    assert gr == case["greedy_bytes_per_p"]
    pl0 = ExactWindow(op, lv, s0, c, (), A.FLAGS_ALL).plan()
    assert _fmt(pl0, s0) == case["exact_saved_p0"]
    if "exact_chosen_p" in case:
        assert A.analyze(op, sites=[c], flags=EXACT).plans[c].p - s0 == case["exact_chosen_p"]
        assert A.analyze(op, sites=[c]).plans[c].p - s0 == case["greedy_chosen_p"]


@pytest.mark.parametrize("seed", range(10))
def test_exact_never_above_greedy_and_equals_bf2(seed):
    txt, _ = random_program(850 + seed, n_body=6, nv=4, ns=2, loop=False)
    op = ir.parse(txt)
    lv = A.liveness(op)
    heads = A.region_heads(op)
    an = A.analyze(op)
    for c in an.sites:
        for p in range(c, heads[c] - 1, -1):
            g = A.plan_window(op, lv, p, c, an.backups, A.FLAGS_ALL)
            e = ExactWindow(op, lv, p, c, an.backups, A.FLAGS_ALL).plan()
            if g is not None:
                assert e is not None and e.payload_bytes <= g.payload_bytes
            bf = brute.BFWindow(op, lv, p, c, an.backups)
            try:
                mn = bf.minimum()
            except ValueError:
                continue
            assert (mn is None) == (e is None)
            if e is not None:
                assert e.payload_bytes == mn[0]
                S = {v for _s, v in e.saved}
                assert bf.feasible_set(S) and S <= bf.preempt_obtainable()


@pytest.mark.parametrize("seed", [815, 832, 850, 867, 953, 997])
def test_exact_plans_replay_poisoned(seed):
    loop = seed % 3 == 0
    txt, size = random_program(seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    an = A.analyze(op, flags=EXACT)
    gr = A.analyze(op)
    assert any(an.plans[c].payload_bytes < gr.plans[c].payload_bytes for c in an.sites)
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    ref, _ = interp.run(an, grid, bufs)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    for _ in range(3):
        sched = [r.integers(0, 40, nw), r.integers(0, 10, nw)]
        out, rec = interp.run(an, grid, bufs, schedule=sched, poison_seed=seed)
        assert rec
        for k in ref:
            if k != "scr":
                assert np.array_equal(out[k], ref[k])


def _parity(txt, flags, policy="EVERY_INSTR"):
    op = ir.parse(txt)
    an = A.analyze(op, policy=policy, flags=flags)
    pol = {"EVERY_INSTR": cb.POLL_EVERY_INSTR, "EXPLICIT": cb.POLL_EXPLICIT}[policy]
    p = cb.Program(txt, flags=flags, poll_policy=pol, debug=cb.DEBUG_NO_COMPILE)
    info = p.info
    assert info["exact_fallback"] == 0 and info["exact_truncated"] == 0
    assert p.backups == an.backups
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c])
    return info


@pytest.mark.parametrize("seed", list(range(12)) + [815, 832, 850, 867])
def test_exact_plan_parity_cpp(seed):
    txt, _ = random_program(seed, loop=seed % 3 == 0, n_body=10)
    _parity(txt, EXACT | (A.FLAG_PRUNE if seed % 4 == 1 else 0))


def test_exact_plan_parity_cpp_fixtures_and_c1():
    for case in json.load(open(os.path.join(GOLD, "exact.json")))["cases"]:
        info = _parity(case["ir"], EXACT)
        assert info["exact_windows"] > 0
    info = _parity(configs.c1()["ir"], EXACT)
    assert info["exact_improved"] > 0          # non-chosen windows


def test_exact_configs_complete_and_never_larger():
    """C++ search completes on every window of the small configs (no
    truncation) and the chosen plans are never larger than greedy's."""
    for txt in (configs.c3_ir(512, 128), configs.c4b_ir(), configs.c2_ir(128, 128, 64)):
        pol = cb.POLL_EXPLICIT if "poll" in txt else cb.POLL_EVERY_INSTR
        g = cb.Program(txt, flags=cb.ALL, poll_policy=pol, debug=cb.DEBUG_NO_COMPILE)
        e = cb.Program(txt, flags=cb.ALL | cb.EXACT, poll_policy=pol, debug=cb.DEBUG_NO_COMPILE)
        assert e.info["exact_truncated"] == 0 and e.info["exact_fallback"] == 0
        for k in range(g.num_sites):
            assert e.site_info(k)["payload_bytes_per_warp"] <= g.site_info(k)["payload_bytes_per_warp"]
