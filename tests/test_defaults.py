"""Defaults ctxb_analyze chooses: the signal path (watcher warp
+ drain notice) and the poll test from the poll-loop cost model, for programs
with flag-mode poll sites.  CPU only (analysis + code generation).

The cost model's input, IR instructions on the shortest CFG loop through a
poll site, is counted here by hand from the IR text in workloads/configs.py:
* C4a (per_lane = 8): `loop:` holds iadd v0 (1), 8 ldg + 7 iadd (15),
  8 shr + 8 iadd (16), iadd s0 / setp / umin / ldg s3 (4), 8 atom.add (8),
  brnz (1) = 45 instructions; one block, its own loop;
* C4b ("edge" polls): `eloop:` setp, brz (2) + `ebody:` iadd, setp, ldg,
  atom.cas, setp, and, atom.add, stg, iadd, bra (10) = 12;
* C1: straight-line, no loop (0).
"""
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from workloads import configs

SIGNAL = cb.WATCHER | cb.DRAIN_NOTICE
TEST_BITS = cb.SYNC_POLL | cb.FLAG_REPLICAS
AUTO_BITS = SIGNAL | TEST_BITS | cb.ARMED_SIGNAL | cb.HOST_SIGNAL


def info(ir, **kw):
    kw["debug"] = kw.get("debug", 0) | cb.DEBUG_NO_COMPILE
    kw.setdefault("poll_policy", cb.POLL_EXPLICIT)
    return cb.Program(ir, **kw).info


@pytest.mark.parametrize("name,ir,loop,test", [
    ("c4a", configs.c4a_ir(1 << 14), 45, cb.SYNC_POLL),
    ("c4b", configs.c4b_ir("edge"), 12, cb.FLAG_REPLICAS),
])
def test_poll_loop_by_hand(name, ir, loop, test):
    i = info(ir)
    assert i["poll_loop_instrs"] == loop
    assert i["flags"] & AUTO_BITS == SIGNAL | test
    assert (loop < cb.DENSE_POLL_INSTRS) == (test == cb.FLAG_REPLICAS)


def test_straight_line_gets_sync_test():
    i = info(configs.c1()["ir"], poll_policy=cb.POLL_EVERY_INSTR)
    assert i["poll_loop_instrs"] == 0
    assert i["flags"] & AUTO_BITS == SIGNAL | cb.SYNC_POLL


@pytest.mark.parametrize("ir", [configs.c2_ir(4096, 4096, 4096, polls="iter"), configs.c2s_ir(),
                                configs.c3_ir(8192, 8192, 64, **configs.BENCH_C3)])
def test_long_loops_get_sync_test(ir):
    i = info(ir)
    assert i["poll_loop_instrs"] >= cb.DENSE_POLL_INSTRS
    assert i["flags"] & AUTO_BITS == SIGNAL | cb.SYNC_POLL


def test_caller_choices_are_kept():
    ir = configs.c2_ir(256, 256, 64, polls="iter")
    base = cb.ALL
    # a chosen signal path: no watcher, the poll test still defaults
    assert info(ir, flags=base | cb.ARMED_SIGNAL)["flags"] & AUTO_BITS == cb.ARMED_SIGNAL | cb.SYNC_POLL
    assert info(ir, flags=base | cb.HOST_SIGNAL)["flags"] & AUTO_BITS == cb.HOST_SIGNAL | cb.SYNC_POLL
    assert info(ir, flags=base | cb.WATCHER)["flags"] & AUTO_BITS == cb.WATCHER | cb.SYNC_POLL
    # a chosen poll test (or a pipelined depth / sparse loads): kept
    assert info(ir, flags=base | cb.FLAG_REPLICAS)["flags"] & TEST_BITS == cb.FLAG_REPLICAS
    assert info(ir, flag_depth=2)["flags"] & TEST_BITS == 0
    assert info(ir, load_every=4)["flags"] & TEST_BITS == 0
    # opt-out, forced mode and polls compiled out: nothing added
    for dbg in (cb.DEBUG_NO_AUTO_SIGNAL, cb.DEBUG_FORCED, cb.DEBUG_NO_POLLS):
        assert info(ir, debug=dbg)["flags"] & AUTO_BITS == 0, dbg


def test_defaults_change_no_plan():
    ir = configs.c4b_ir("both")
    a = cb.Program(ir, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
    b = cb.Program(ir, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_AUTO_SIGNAL)
    assert [a.plan_text(k) for k in range(a.num_sites)] == [b.plan_text(k) for k in range(b.num_sites)]
    assert "warp_exit(P, lane, &blk_out)" in a.source and "#define CTXB_NOTICE_HOST 1" in a.source
    assert "#define CTXB_NOTICE_HOST 0" in b.source
