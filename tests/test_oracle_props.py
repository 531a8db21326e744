"""Property pins of the oracle on seeded random IR programs.

* liveness == a path-search definition of liveness (textbook, brute force);
* sufficiency: preempt at random poll visits (nested, two
  launches), poison every register, restore + replay -> final memory equals
  the uninterrupted run;
* p = c is always a flashback-point; bytes(CTXBack) <= bytes(LIVE) <= FULL_IR;
* with all techniques off the feasible set is exactly the basic condition
  "no register of R_prec overwritten by [I_prec, I_cur)";
* straight-line code without redefinitions: closed-form context per p;
* BF2: every oracle plan's saved set is sufficient (closure) and never
  smaller than the exhaustive minimum; oracle-feasible => BF-feasible;
* BF3: the chosen p is the lexicographic minimum over all p (R-10).
"""
import numpy as np
import pytest

from oracle import analysis as A
from oracle import brute, interp, ir
from workloads.randprog import random_buffers, random_program


def prog_for(seed, **kw):
    loop = kw.pop("loop", seed % 3 == 0)
    txt, size = random_program(seed, loop=loop, **kw)
    p = ir.parse(txt)
    nout = p.nv - 1 + (p.ns - (1 if loop else 0))
    return p, size, nout


def instr_succ(prog, i):
    ins = prog.instrs[i]
    lab = {k: prog.bbs[b][0] for k, b in prog.labels.items()}
    if ins.op == "exit":
        return []
    if ins.op == "bra":
        return [lab[ins.target]]
    if ins.op in ("brnz", "brz"):
        return [i + 1, lab[ins.target]]
    return [i + 1]


def live_by_paths(prog, i, r):
    """r is live before i iff some path from i reads r before writing it."""
    seen = set()
    stack = [i]
    while stack:
        k = stack.pop()
        if k in seen:
            continue
        seen.add(k)
        ins = prog.instrs[k]
        if r in ins.uses():
            return True
        if ins.defreg == r:
            continue
        stack.extend(instr_succ(prog, k))
    return False


@pytest.mark.parametrize("seed", range(12))
def test_liveness_matches_path_definition(seed):
    p, _size, _n = prog_for(seed, n_body=8)
    lv = A.liveness(p)
    for i in range(len(p.instrs)):
        for r in p.all_regs():
            assert (r in lv.live_in[i]) == live_by_paths(p, i, r), (seed, i, r)


@pytest.mark.parametrize("seed", range(40))
def test_sufficiency_random_nested_preemption(seed):
    p, size, nout = prog_for(seed, n_body=10)
    an = A.analyze(p)
    grid = 2
    bufs = random_buffers(seed, p.block, grid, size, nout)
    ref, _ = interp.run(an, grid, bufs)
    rng = np.random.default_rng(1000 + seed)
    nw = grid * p.nwarps
    for _trial in range(4):
        sched = [rng.integers(0, 40, nw), rng.integers(0, 40, nw), rng.integers(0, 10, nw)]
        out, rec = interp.run(an, grid, bufs, schedule=sched, poison_seed=seed)
        for k in ref:
            if k == "scr":        # racy scratch buffer (same index from every block)
                continue
            assert np.array_equal(out[k], ref[k]), (seed, k)
        for r in rec:
            pl = an.live[r["site"]] if r["kind"] == "live" else an.plans[r["site"]]
            assert r["bytes"] == pl.payload_bytes


@pytest.mark.parametrize("seed", range(40))
def test_ordering_invariants(seed):
    p, _size, _n = prog_for(seed, n_body=10)
    an = A.analyze(p)
    full = A.full_ir_bytes(p)
    for c in an.sites:
        assert A.plan_window(p, an.lv, c, c, an.backups) is not None
        assert an.plans[c].payload_bytes <= an.live[c].payload_bytes <= full
        assert an.live[c].payload_bytes == sum(128 if r[0] == "v" else 4 for r in an.lv.live_in[c])


@pytest.mark.parametrize("seed", range(20))
def test_basic_condition(seed):
    p, _size, _n = prog_for(seed, n_body=8)
    lv = A.liveness(p)
    heads = A.region_heads(p)
    for c in range(len(p.instrs)):
        for q in range(heads[c], c + 1):
            pl = A.plan_window(p, lv, q, c, (), 0)
            overwritten = any(p.instrs[j].defreg in lv.live_in[q] for j in range(q, c)
                              if p.instrs[j].defreg)
            reexec_all = all(A.reexec_op_kind(p, p.instrs[j]) for j in range(q, c) if p.instrs[j].defreg)
            assert (pl is not None) == (not overwritten and reexec_all)
            if pl is not None:
                assert pl.payload_bytes == sum(128 if r[0] == "v" else 4 for r in lv.live_in[q])


def test_straight_line_no_redefinition_closed_form():
    """Every instruction defines a fresh register and all are ALU ops, so every
    value is CURRENT at I_cur and every live-out result is re-executable.  Then
    (R-2) the context of flashback-point p is the set of registers
    defined before p that are read by a live-out instruction of [p, c) or are
    live-in at c, and resume re-executes exactly the live-out instructions.
    The chosen p minimises (bytes, #re-executions, -p) (R-10)."""
    rng = np.random.default_rng(77)
    for trial in range(40):
        n = 14
        lines = [".kernel sl", ".buffer ro a", ".buffer wo o", f".vregs {n + 3}", ".sregs 0", ".block 32",
                 "init:", "  ldg v0, a[%tid]", "  ldg v1, a[%laneid]", "  ldg v2, a[%tid]", "  bra m", "m:"]
        for k in range(3, n + 3):
            a, b = rng.integers(0, k, 2)
            op = ["iadd", "xor", "imul", "and", "shl", "fadd"][int(rng.integers(6))]
            lines.append(f"  {op} v{k}, v{a}, v{b}")
        outs = sorted(set(int(x) for x in rng.integers(0, n + 3, 4)))
        for o in outs:
            lines.append(f"  stg o[v{o}], v{o}")
        lines.append("  exit")
        p = ir.parse("\n".join(lines) + "\n")
        lv = A.liveness(p)
        s0 = p.bbs[p.labels["m"]][0]
        c = s0 + n
        an = A.analyze(p, sites=[c], keep_candidates=True)
        costs = {}
        for q in range(s0, c + 1):
            before = {"v0", "v1", "v2"} | {p.instrs[j].defreg for j in range(s0, q)}
            live_j = [j for j in range(q, c) if p.instrs[j].defreg in lv.live_out[j]]
            need = set()
            for j in live_j:
                need |= set(p.instrs[j].uses()) & before
            need |= set(lv.live_in[c]) & before
            costs[q] = (128 * len(need), 0, len(live_j), -q)
            assert an.candidates[c][q].cost() == costs[q]
        best = min(costs.values())
        assert an.plans[c].cost() == best


@pytest.mark.parametrize("seed", range(25))
def test_bf2_soundness_and_minimum(seed):
    p, _size, _n = prog_for(seed, n_body=5, nv=4, ns=2, mem_ops=True, fp=False, loop=False)
    lv = A.liveness(p)
    an = A.analyze(p)
    heads = an.heads
    checked = 0
    for c in an.sites:
        if c - heads[c] > 8:
            continue
        for q in range(heads[c], c + 1):
            try:
                r = brute.check_window(p, lv, q, c, an.backups)
            except ValueError:
                continue
            checked += 1
            if r["oracle_feasible"]:
                assert r["bf_feasible"]
                assert r["sound"]
                assert r["oracle_bytes"] >= r["bf_bytes"]
    assert checked > 0


@pytest.mark.parametrize("seed", range(10))
def test_bf3_chosen_is_lexicographic_min(seed):
    p, _size, _n = prog_for(seed, n_body=8)
    an = A.analyze(p, keep_candidates=True)
    for c in an.sites:
        feas = [pl for pl in an.candidates[c].values() if pl is not None]
        assert an.plans[c].cost() == min(pl.cost() for pl in feas)
        assert sorted(an.candidates[c]) == list(range(an.heads[c], c + 1))


@pytest.mark.parametrize("rows", [1, 2, 4])
def test_c3_oracle_equals_textbook_stencil_under_preemption(rows):
    """Pin for the C3 workload as the bench runs it (rows_per_iter = 2): the
    oracle interpreter's output equals a plain numpy 5-point stencil in the
    IR's f32 operation order, uninterrupted and under random nested forced
    preemption with poisoned registers, for 1, 2 and 4 rows per iteration."""
    from workloads import configs
    W, H = 512, 64
    cfg = configs.c3(W, H, 32, rows_per_iter=rows)
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT")
    grid = (W // 256) * (H // 32)
    want = configs.c3_numpy_reference(cfg["buffers"]["X"], W, H)
    out, _ = interp.run(an, grid, cfg["buffers"])
    assert np.array_equal(out["Y"], want)
    r = np.random.default_rng(40 + rows)
    nw = grid * op.nwarps
    for _ in range(3):
        sched = [r.integers(0, 40 // rows, nw).astype(np.uint32), r.integers(0, 8, nw).astype(np.uint32)]
        out, rec = interp.run(an, grid, cfg["buffers"], schedule=sched, poison_seed=rows)
        assert rec and np.array_equal(out["Y"], want)
