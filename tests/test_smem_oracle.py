"""NEXT N2 on the CPU: shared memory + barriers in the IR, both parsers, the
analysis rules (lds not re-executable, `bar` ends the idempotent region,
barrier kernels preempt only at barriers), and the oracle's block-uniform
preemption (smem slices saved, poisoned, restored)."""
import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import interp, ir
from workloads import configs

SMEM_K = """.kernel rev
.buffer ro a
.buffer wo o
.vregs 4
.sregs 1
.block 64
.smem 64
  ldg v0, a[%tid]
  imul v1, v0, 3
  sts %tid, v1
  bar
  isub v2, 63, %tid
  lds v3, v2
  iadd v3, v3, v0
  bar
  sts %tid, v3
  bar
  lds v2, v2
  xor v2, v2, v1
  stg o[%tid], v2
  exit
"""


def test_parsers_accept_and_reject_the_same():
    ir.parse(SMEM_K)
    cb.Program(SMEM_K, debug=cb.DEBUG_NO_COMPILE)
    bad = [SMEM_K.replace(".smem 64\n", ""),                           # lds/sts without .smem
           SMEM_K.replace("  bar\n", ""),                              # smem without barriers
           SMEM_K.replace("  isub v2, 63, %tid", "  poll\n  isub v2, 63, %tid")]   # poll not at a bar
    for t in bad:
        with pytest.raises(ir.IRError):
            ir.parse(t)
        with pytest.raises(cb.CtxbError) as e:
            cb.Program(t, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
        assert e.value.code == -2


def test_barrier_kernel_sites_and_rules():
    op = ir.parse(SMEM_K)
    an = A.analyze(op)
    assert [op.instrs[c].op for c in an.sites] == ["bar", "bar", "bar"]
    heads = A.region_heads(op)
    bars = [i for i, x in enumerate(op.instrs) if x.op == "bar"]
    for c in range(len(op.instrs)):
        prev = [b for b in bars if b < c]
        assert heads[c] >= (prev[-1] + 1 if prev else 0)
    lds = [i for i, x in enumerate(op.instrs) if x.op == "lds"]
    assert not any(A.reexec_op_kind(op, op.instrs[i]) for i in lds)
    p = cb.Program(SMEM_K, debug=cb.DEBUG_NO_COMPILE)
    assert p.num_sites == 3
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c])


def test_block_uniform_preemption_replays():
    op = ir.parse(SMEM_K)
    an = A.analyze(op)
    r = np.random.default_rng(0)
    bufs = {"a": r.integers(0, 1 << 32, 64, dtype=np.uint64).astype(np.uint32), "o": np.zeros(256, np.uint32)}
    ref, _ = interp.run(an, 3, bufs)
    # textbook check of the kernel itself
    a = bufs["a"]
    tid = np.arange(64)
    s1 = (a * np.uint32(3)).astype(np.uint32)
    s2 = (s1[63 - tid] + a).astype(np.uint32)
    want = (s2[63 - tid] ^ s1).astype(np.uint32)
    assert np.array_equal(ref["o"][:64], want)
    for t in range(4):
        sched = [r.integers(0, 3, 6), r.integers(0, 2, 6)]
        out, rec = interp.run(an, 3, bufs, schedule=sched, poison_seed=t)
        assert np.array_equal(out["o"], ref["o"])
        by_launch = {}
        for x in rec:
            by_launch.setdefault((x["launch"], x["warp"] // 2), []).append(x)
        assert all(len(v) == 2 for v in by_launch.values())            # both warps of the block
        assert all(x["bytes"] == an.plans[x["site"]].payload_bytes + 4 * 32 for x in rec
                   if x["kind"] != "live")


def test_c2s_equals_c2_in_the_oracle():
    c2s = configs.c2s(128, 128, 16)
    c2 = configs.c2(128, 128, 16)
    a1 = A.analyze(ir.parse(c2s["ir"]), policy="EXPLICIT")
    a2 = A.analyze(ir.parse(c2["ir"]), policy="EXPLICIT")
    o1, _ = interp.run(a1, 1, c2s["buffers"])
    o2, _ = interp.run(a2, 1, c2["buffers"])
    assert np.array_equal(o1["C"], o2["C"])
