"""Demand-driven restore (NEXT N4, `CTXB_PRUNE`): only the values the
registers live at I_cur need are restored (instead of every live-out result
of the window, R-2 literal).  Pins: poisoned replays stay exact; the pruned
context is never larger than the literal one; it is sufficient by the BF2
closure with the required set = the final values of LIVE_IN(c); C++ plans
equal the oracle's."""
import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import brute, interp, ir
from workloads import configs
from workloads.randprog import random_buffers, random_program

PRUNE = A.FLAGS_ALL | A.FLAG_PRUNE


@pytest.mark.parametrize("seed", range(20))
def test_prune_plan_parity(seed):
    txt, _ = random_program(500 + seed, loop=seed % 3 == 0, n_body=10)
    op = ir.parse(txt)
    an = A.analyze(op, flags=PRUNE)
    p = cb.Program(txt, flags=cb.ALL | cb.PRUNE, debug=cb.DEBUG_NO_COMPILE)
    assert p.backups == an.backups
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c])


@pytest.mark.parametrize("seed", range(20))
def test_prune_replays_and_never_larger(seed):
    loop = seed % 3 == 0
    txt, size = random_program(500 + seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    an = A.analyze(op, flags=PRUNE)
    lit = A.analyze(op)
    for c in an.sites:
        assert an.plans[c].payload_bytes <= lit.plans[c].payload_bytes
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    ref, _ = interp.run(an, grid, bufs)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    for _ in range(3):
        sched = [r.integers(0, 40, nw), r.integers(0, 10, nw)]
        out, rec = interp.run(an, grid, bufs, schedule=sched, poison_seed=seed)
        for k in ref:
            if k != "scr":
                assert np.array_equal(out[k], ref[k])


def test_prune_unblocks_dead_chains():
    """The paper's literal rule blocks a window whose dead intermediate chain
    lost an input (e.g. a rolling register overwritten by a MOV); pruning
    restores only what I_cur needs, so the context can only shrink."""
    op = ir.parse(configs.c2_ir(128, 128, 16, polls="half"))
    lit = A.analyze(op, policy="EXPLICIT")
    pr = A.analyze(op, policy="EXPLICIT", flags=PRUNE)
    tot_l = sum(lit.plans[c].payload_bytes for c in lit.sites)
    tot_p = sum(pr.plans[c].payload_bytes for c in pr.sites)
    assert tot_p <= tot_l


@pytest.mark.parametrize("seed", range(12))
def test_prune_bf2_sufficiency(seed):
    txt, _ = random_program(600 + seed, n_body=5, nv=4, ns=2, fp=False, loop=False)
    op = ir.parse(txt)
    lv = A.liveness(op)
    an = A.analyze(op, flags=PRUNE)
    for c in an.sites:
        pl = an.plans[c]
        bf = brute.BFWindow(op, lv, pl.p, c, an.backups)
        req = set()
        for r in lv.live_in[c]:
            req.add((r, bf.w.rd(r, c)))
        S = {v for _s, v in pl.saved}
        assert req <= bf.closure(S)
        assert S <= bf.preempt_obtainable()
