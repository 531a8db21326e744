"""Combined preempt + resume ranking (NEXT N4, `CTXB_RANK_RESUME`).

The paper picks the flashback-point with the least preemption latency (P:313,
P:337) and notes that re-execution can dominate resuming.  With
the flag each site picks the candidate minimising

    E = 2 * payload + re-executed load bytes + level_bytes * (levels - 1)
      + instr_bytes * (#reverts + #re-executions)

(DESIGN.md §8e), ties by the R-10 key.  Pins: hand-computed E of every
candidate of a dependent-load chain; the paper's ALU-only figures keep their
choice (E from the golden plans); poisoned replays stay exact; C++ plans equal
the oracle's.
"""
import json
import os

import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import interp, ir
from workloads import configs
from workloads.randprog import random_buffers, random_program

RANK = A.FLAGS_ALL | A.FLAG_RANK_RESUME
GOLD = os.path.join(os.path.dirname(__file__), "golden")

# I0 mov v0,%tid; I1 ldg v1,X[v0]; I2 ldg v2,X[v1]; I3 iadd v3,v2,1; site c = I4.
CHAIN = """\
.kernel chain
.buffer ro X
.buffer wo Y
.vregs 4
.sregs 0
.block 32
main:
  mov v0, %tid
  ldg v1, X[v0]
  ldg v2, X[v1]
  iadd v3, v2, 1
  stg Y[v0], v3
  exit
"""

# Hand derivation (LIVE_IN(I4) = {v0, v3}; instr_bytes 8, level_bytes 512):
#   p=4  LIVE: save v0,v3                  E = 2*256                          = 512
#   p=3  save v0,v2; re-exec I3 (level 1)  E = 2*256 + 8                      = 520
#   p=2  save v0,v1; I2 load at level 2    E = 2*256 + 128 + 512*1 + 8*2      = 1168
#   p=1  save v0; loads at levels 2, 3     E = 2*128 + 256 + 512*2 + 8*3      = 1560
#   p=0  save nothing; I0 level 0, loads 1, 2  E = 0 + 256 + 512*1 + 8*4      = 800
CHAIN_E = {4: 512, 3: 520, 2: 1168, 1: 1560, 0: 800}
CHAIN_BYTES = {4: 256, 3: 256, 2: 256, 1: 128, 0: 0}


def test_chain_estimates_by_hand():
    op = ir.parse(CHAIN)
    lv = A.liveness(op)
    for p, e in CHAIN_E.items():
        pl = A.plan_window(op, lv, p, 4)
        assert pl is not None and pl.payload_bytes == CHAIN_BYTES[p]
        assert A.resume_estimate(op, pl) == e, p


@pytest.mark.parametrize("level_bytes,expect_p", [(512, 4), (300, 4), (200, 0), (64, 0)])
def test_chain_choice_moves_with_level_weight(level_bytes, expect_p):
    """E(p=0) = 288 + level_bytes vs E(LIVE) = 512: the chain is re-executed
    only when a dependent round trip is cheaper than 224 context bytes."""
    op = ir.parse(CHAIN)
    an = A.analyze(op, sites=[4], flags=RANK, resume_level_bytes=level_bytes)
    assert an.plans[4].p == expect_p
    assert A.analyze(op, sites=[4]).plans[4].p == 0          # R-10: least bytes
    p = cb.Program(CHAIN, flags=cb.ALL | cb.RANK_RESUME, resume_level_bytes=level_bytes,
                   debug=cb.DEBUG_NO_COMPILE)
    assert p.site_info(4)["p"] == expect_p


@pytest.mark.parametrize("name", ["fig2", "fig3", "fig4", "fig6"])
def test_paper_figures_keep_their_choice(name):
    """ALU-only windows: E = 2*bytes + 8*ops, so the paper's least-context
    choice stays (E computed from the golden plan, not from the oracle)."""
    g = json.load(open(os.path.join(GOLD, name + ".json")))
    prog = ir.parse(g["ir"])
    s0 = prog.bbs[prog.labels["main"]][0]
    c = s0 + g["site"]
    an = A.analyze(prog, sites=[c], flags=RANK)
    pl = an.plans[c]
    assert pl.p - s0 == g["chosen_p"]
    ops = len(g["reexec"]) + len(g["revert_pre"]) + len(g["revert_res"])
    assert A.resume_estimate(prog, pl) == 2 * A.VEC_BYTES * len(g["saved"]) + 8 * ops


@pytest.mark.parametrize("seed", range(20))
def test_rank_plan_parity(seed):
    txt, _ = random_program(700 + seed, loop=seed % 3 == 0, n_body=10)
    op = ir.parse(txt)
    lb = (64, 512, 4096)[seed % 3]
    an = A.analyze(op, flags=RANK | (A.FLAG_PRUNE if seed % 2 else 0), resume_level_bytes=lb)
    p = cb.Program(txt, flags=cb.ALL | cb.RANK_RESUME | (cb.PRUNE if seed % 2 else 0), resume_level_bytes=lb,
                   debug=cb.DEBUG_NO_COMPILE)
    assert p.backups == an.backups
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c])


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4a", "c4b"])
def test_rank_config_parity(name):
    txt = {"c1": lambda: configs.c1()["ir"], "c2": lambda: configs.c2_ir(128, 128, 64),
           "c3": lambda: configs.c3_ir(512, 128), "c4a": lambda: configs.c4a_ir(1 << 14),
           "c4b": configs.c4b_ir}[name]()
    pol = "EVERY_INSTR" if name == "c1" else "EXPLICIT"
    op = ir.parse(txt)
    an = A.analyze(op, policy=pol, flags=RANK)
    base = A.analyze(op, policy=pol)
    p = cb.Program(txt, flags=cb.ALL | cb.RANK_RESUME, poll_policy=getattr(cb, "POLL_" + pol),
                   debug=cb.DEBUG_NO_COMPILE)
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c])
        # the chosen E never exceeds the R-10 choice's or LIVE's
        e = A.resume_estimate(op, an.plans[c])
        assert e <= A.resume_estimate(op, base.plans[c])
        assert e <= A.resume_estimate(op, an.live[c])


def test_rank_moves_c3_to_live():
    """C3: the R-10 choice re-executes five row loads after restoring the
    index (two memory levels); the combined ranking keeps the loaded values."""
    op = ir.parse(configs.c3_ir(512, 128))
    an = A.analyze(op, policy="EXPLICIT", flags=RANK)
    base = A.analyze(op, policy="EXPLICIT")
    for c in an.sites:
        assert base.plans[c].p < c and an.plans[c].p == c


@pytest.mark.parametrize("seed", range(12))
def test_rank_replays(seed):
    loop = seed % 3 == 0
    txt, size = random_program(700 + seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    an = A.analyze(op, flags=RANK, resume_level_bytes=(64, 512, 4096)[seed % 3])
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    ref, _ = interp.run(an, grid, bufs)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    for _ in range(3):
        sched = [r.integers(0, 40, nw), r.integers(0, 10, nw)]
        out, _rec = interp.run(an, grid, bufs, schedule=sched, poison_seed=seed)
        for k in ref:
            if k != "scr":
                assert np.array_equal(out[k], ref[k])
