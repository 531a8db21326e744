"""CS-Defer and CTXBack+CS-Defer, NEXT item N1.

CPU: the C++ analyzer's deferral targets equal the oracle's; every target is
a later site of the same basic block whose estimated latency is no larger
than saving at the site itself; preemptions carried to their target replay
correctly under poison (the sufficiency lemma, holds at the target).
"""
import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import interp, ir
from workloads import configs
from workloads.randprog import random_buffers, random_program


@pytest.mark.parametrize("mode", [A.MODE_CTXBACK, A.MODE_LIVE])
@pytest.mark.parametrize("seed", range(12))
def test_defer_targets_parity(seed, mode):
    txt, _ = random_program(300 + seed, loop=seed % 2 == 0, n_body=10)
    op = ir.parse(txt)
    an = A.analyze(op, mode=mode, flags=A.FLAGS_ALL | A.FLAG_DEFER)
    p = cb.Program(txt, flags=cb.ALL | cb.DEFER, mode=mode, debug=cb.DEBUG_NO_COMPILE)
    assert [p.site_info(k)["defer_site"] for k in range(p.num_sites)] == \
        [an.sites.index(an.defer[c]) for c in an.sites]


@pytest.mark.parametrize("instr_bytes", [1, 8, 64])
def test_defer_targets_are_estimate_minima(instr_bytes):
    op = ir.parse(configs.c1()["ir"])
    an = A.analyze(op, flags=A.FLAGS_ALL | A.FLAG_DEFER, defer_instr_bytes=instr_bytes)
    for c in an.sites:
        d = an.defer[c]
        assert d >= c and op.bb_of(d) == op.bb_of(c)
        est = lambda x: an.plans[x].payload_bytes + instr_bytes * (x - c)  # noqa: E731
        later = [x for x in an.sites if x >= c and op.bb_of(x) == op.bb_of(c)]
        assert est(d) == min(est(x) for x in later)
        assert all(est(x) > est(d) for x in later if x < d)     # earliest minimum
    p = cb.Program(configs.c1()["ir"], flags=cb.ALL | cb.DEFER, defer_instr_bytes=instr_bytes,
                   debug=cb.DEBUG_NO_COMPILE)
    assert [p.site_info(k)["defer_site"] for k in range(p.num_sites)] == \
        [an.sites.index(an.defer[c]) for c in an.sites]


@pytest.mark.parametrize("mode", [A.MODE_CTXBACK, A.MODE_LIVE])
@pytest.mark.parametrize("seed", range(10))
def test_deferred_preemption_replays(seed, mode):
    loop = seed % 3 == 0
    txt, size = random_program(400 + seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    an = A.analyze(op, mode=mode, flags=A.FLAGS_ALL | A.FLAG_DEFER, defer_instr_bytes=2)
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    ref, _ = interp.run(an, grid, bufs)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    deferred = 0
    for _ in range(4):
        sched = [r.integers(0, 40, nw), r.integers(0, 10, nw)]
        out, rec = interp.run(an, grid, bufs, schedule=sched, poison_seed=seed)
        for k in ref:
            if k != "scr":
                assert np.array_equal(out[k], ref[k])
        for x in rec:
            pl = an.live[x["site"]] if x["kind"] == "live" else an.plans[x["site"]]
            assert x["bytes"] == pl.payload_bytes
        deferred += sum(1 for c in an.sites if an.defer[c] != c)
    assert deferred > 0
