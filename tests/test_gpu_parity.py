"""GPU parity: the generated sm_100a kernels (through the C-ABI) against the
oracle, on the same seeded inputs, element by element.

* uninterrupted outputs are bit-exact with the oracle interpreter;
* forced preemption at every site / random per-warp sites / nested
  re-preemption: final outputs bit-exact with the uninterrupted run and the
  oracle, and every preempted warp's header (site, LIVE-fallback flag,
  payload bytes) equals the oracle's record (context bytes == oracle's);
* the same with the poison debug mode (every IR register of a resumed warp
  starts as garbage, so a plan that relies on an unsaved register fails).
"""
import numpy as np
import pytest

from oracle import analysis as A
from oracle import interp, ir
from workloads import configs
from workloads.randprog import random_buffers, random_program

from gpu_helpers import gpu_run, header_records, oracle_records

pytestmark = pytest.mark.gpu


def _cb():
    import paper_conf_ipps_jiw21_b200 as cb
    return cb


def check(txt, grid, bufs, schedules, policy="EVERY_INSTR", skip=("scr",), poison=True, flags=7, mode=0,
          defer_instr_bytes=8, runtime_flags=0):
    cb = _cb()
    op = ir.parse(txt)
    an = A.analyze(op, policy=policy, flags=flags, mode=mode, defer_instr_bytes=defer_instr_bytes)
    pol = {"EVERY_INSTR": cb.POLL_EVERY_INSTR, "EXPLICIT": cb.POLL_EXPLICIT}[policy]
    dbg = cb.DEBUG_FORCED | (cb.DEBUG_POISON if poison else 0)
    prog = cb.Program(txt, flags=flags | runtime_flags, poll_policy=pol, debug=dbg, mode=mode,
                      defer_instr_bytes=defer_instr_bytes)
    names = list(op.buffers)
    ref, _ = interp.run(an, grid, bufs)
    g0, h0, _ = gpu_run(prog, names, grid, bufs, {})
    for n in names:
        if n in skip:
            continue
        assert np.array_equal(g0[n], ref[n]), f"uninterrupted output {n} differs from the oracle"
    for sched in schedules:
        out, rec = interp.run(an, grid, bufs, schedule=sched)
        g, hdrs, run = gpu_run(prog, names, grid, bufs, {}, schedule=sched)
        for n in names:
            if n in skip:
                continue
            assert np.array_equal(g[n], ref[n]), f"{n} after preempt/resume differs (schedule {sched})"
            assert np.array_equal(out[n], ref[n])
        assert header_records(hdrs) [:len(oracle_records(rec, an))] == oracle_records(rec, an)
    return prog, an


def test_c1_every_site_all_warps():
    cfg = configs.c1()
    scheds = [[[k] * 4] for k in range(24)]
    check(cfg["ir"], 1, cfg["buffers"], scheds)


def test_c1_random_per_warp_sites_and_nested():
    cfg = configs.c1()
    vecs = configs.c1_random_site_vectors(512)
    r = np.random.default_rng(8)
    scheds = []
    for i, v in enumerate(vecs):
        if i % 4 == 0:   # nested: re-preempt after the resume (LIVE fallback in the same BB pass)
            scheds.append([v, r.integers(0, 6, 4).astype(np.uint32)])
        else:
            scheds.append([v])
    check(cfg["ir"], 1, cfg["buffers"], scheds)


def test_c1_bytes_equal_oracle_per_site():
    cb = _cb()
    cfg = configs.c1()
    op = ir.parse(cfg["ir"])
    an = A.analyze(op)
    prog = cb.Program(cfg["ir"], debug=cb.DEBUG_NO_COMPILE)
    for k, c in enumerate(an.sites):
        si = prog.site_info(k)
        assert si["payload_bytes_per_warp"] == an.plans[c].payload_bytes
        assert si["p"] == an.plans[c].p
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])


@pytest.mark.parametrize("seed", range(12))
def test_random_programs(seed):
    loop = seed % 3 == 0
    txt, size = random_program(seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    grid = 3
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 60, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)] for _ in range(6)]
    check(txt, grid, bufs, scheds)


@pytest.mark.parametrize("seed", range(6))
def test_random_loop_nests(seed):
    """Loop nests: resumes inside the inner and the outer loop
    go through RT_k and the peeled copy of the nest; forced, nested, poisoned."""
    txt, size = random_program(700 + seed, loop=True, nested=True, n_body=8)
    op = ir.parse(txt)
    grid = 2
    nout = op.nv - 1 + op.ns - 2
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 90, nw).astype(np.uint32), r.integers(0, 40, nw).astype(np.uint32)] for _ in range(6)]
    check(txt, grid, bufs, scheds)


@pytest.mark.parametrize("seed,indexed", [(s, 1 + s % 2) for s in range(6)])
def test_random_indexed_loops(seed, indexed):
    """Loop-carried index bases: resumed iterations run the fast
    path (bases < 2^31, masked) or, with a top-bit-set base whose `+ c` wraps
    into range, the generic path; forced, nested, poisoned; bit-exact."""
    txt, size = random_program(800 + seed, loop=True, nested=seed % 3 == 0, indexed=indexed, n_body=10)
    op = ir.parse(txt)
    grid = 2
    bufs = random_buffers(seed, op.block, grid, size, txt.count("stg out["))
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 90, nw).astype(np.uint32), r.integers(0, 40, nw).astype(np.uint32)] for _ in range(6)]
    check(txt, grid, bufs, scheds)


@pytest.mark.parametrize("name", ["fig2", "fig3", "fig4", "fig5", "fig6", "r9", "r3", "r3bar", "osrb_select", "n3"])
def test_paper_figures_on_gpu(name):
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", name + ".json")))
    op = ir.parse(g["ir"])
    r = np.random.default_rng(3)
    bufs = {b: (r.integers(0, 64, 64, dtype=np.uint32) if k == "ro" else np.zeros(64, np.uint32))
            for b, k in op.buffers.items()}
    n = len(op.instrs)
    check(g["ir"], 1, bufs, [[[k]] for k in range(n)])


@pytest.mark.parametrize("mode", [0, 1])
def test_c1_cs_defer(mode):
    """CS-Defer (mode LIVE + DEFER) and CTXBack+CS-Defer (CTXBACK + DEFER):
    preemptions carried to their deferral target, bit-exact, bytes = oracle."""
    cfg = configs.c1()
    vecs = configs.c1_random_site_vectors(64, seed=9)
    scheds = [[[k] * 4] for k in range(24)] + [[v] for v in vecs]
    check(cfg["ir"], 1, cfg["buffers"], scheds, flags=15, mode=mode)


@pytest.mark.parametrize("seed", range(6))
def test_random_programs_defer(seed):
    loop = seed % 3 == 0
    txt, size = random_program(400 + seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 60, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)] for _ in range(4)]
    check(txt, grid, bufs, scheds, flags=15, mode=seed % 2, defer_instr_bytes=2)


@pytest.mark.parametrize("seed", range(6))
def test_random_programs_prune(seed):
    """Demand-driven restore (CTXB_PRUNE, NEXT N4) on the GPU vs the oracle."""
    loop = seed % 3 == 0
    txt, size = random_program(500 + seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 60, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)] for _ in range(4)]
    check(txt, grid, bufs, scheds, flags=23)


@pytest.mark.parametrize("seed", range(6))
def test_random_programs_rank_resume(seed):
    """Combined preempt + resume ranking (CTXB_RANK_RESUME, NEXT N4) on the GPU."""
    loop = seed % 3 == 0
    txt, size = random_program(700 + seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 60, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)] for _ in range(4)]
    check(txt, grid, bufs, scheds, flags=7 | 32 | (16 if seed % 2 else 0))


def test_c2_half_prune_small():
    cfg = configs.c2(128, 128, 32, polls="half")
    r = np.random.default_rng(2)
    scheds = [[r.integers(0, 64, 8).astype(np.uint32), r.integers(0, 8, 8).astype(np.uint32)] for _ in range(3)]
    check(cfg["ir"], 1, cfg["buffers"], scheds, policy="EXPLICIT", flags=23)


def test_smem_barrier_kernel_block_uniform():
    """NEXT N2 on the GPU: shared memory + barriers, block-uniform preemption
    at the barriers (forced per-warp targets OR-ed per block), nested."""
    import sys, os
    sys.path.insert(0, os.path.dirname(__file__))
    from test_smem_oracle import SMEM_K
    r = np.random.default_rng(1)
    bufs = {"a": r.integers(0, 1 << 32, 64, dtype=np.uint64).astype(np.uint32), "o": np.zeros(256, np.uint32)}
    scheds = [[[k] * 6] for k in range(3)] + [[r.integers(0, 3, 6).astype(np.uint32),
                                               r.integers(0, 2, 6).astype(np.uint32)] for _ in range(6)]
    check(SMEM_K, 3, bufs, scheds)


@pytest.mark.parametrize("seed", [815, 832, 850, 867, 953, 997])
def test_random_programs_exact(seed):
    """Exact minimum-bytes plans (CTXB_EXACT, NEXT N4) on the GPU vs the oracle;
    the seeds are programs where the exact plan beats greedy at >= 1 site."""
    loop = seed % 3 == 0
    txt, size = random_program(seed, loop=loop, n_body=10)
    op = ir.parse(txt)
    grid = 2
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    n = len(op.instrs)
    scheds = [[[k] * nw] for k in range(0, n, 3)] + \
             [[r.integers(0, 60, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)] for _ in range(4)]
    check(txt, grid, bufs, scheds, flags=7 | 64 | (16 if seed % 2 else 0))


@pytest.mark.parametrize("k", [0, 1])
def test_exact_fixtures_and_c1_on_gpu(k):
    import json
    import os
    if k == 0:
        cfg = configs.c1()
        check(cfg["ir"], 1, cfg["buffers"], [[[s] * 4] for s in range(24)], flags=7 | 64)
    for case in json.load(open(os.path.join(os.path.dirname(__file__), "golden", "exact.json")))["cases"]:
        op = ir.parse(case["ir"])
        r = np.random.default_rng(5 + k)
        bufs = {b: (r.integers(0, 1 << 32, 64, dtype=np.uint64).astype(np.uint32) if kd == "ro"
                    else np.zeros(64, np.uint32)) for b, kd in op.buffers.items()}
        check(case["ir"], 1, bufs, [[[s]] for s in range(len(op.instrs))], flags=7 | 64)   # 1 block: outputs indexed by %tid


def test_c1_gather_resume_nested():
    """CTXB_GATHER_RESUME with forced nested preemption and poison (C1)."""
    cfg = configs.c1()
    vecs = configs.c1_random_site_vectors(64, seed=11)
    scheds = [[[k] * 4] for k in range(0, 24, 2)] + [[v, v // 2] for v in vecs[:32]]
    check(cfg["ir"], 1, cfg["buffers"], scheds, flags=7 | 128)


@pytest.mark.parametrize("slot", ["smem", "lanes"])
@pytest.mark.parametrize("seed", range(8))
def test_osrb_smem_slots(seed, slot):
    """CTXB_OSRB_SMEM / CTXB_OSRB_LANES: the same plans with OSRB backups in
    per-warp shared-memory slots (the paper's LDS tier) or in the lanes of one
    register (the VGPR-lane tier); poisoned forced and nested
    preemption bit-exact, headers = oracle.  Seed 0 is the paper's Fig. 5
    OSRB example; the others are random loop programs."""
    rf = _cb().OSRB_SMEM if slot == "smem" else _cb().OSRB_LANES
    import json
    import os
    if seed == 0:
        g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fig5.json")))
        op = ir.parse(g["ir"])
        r = np.random.default_rng(3)
        bufs = {b: (r.integers(0, 64, 64, dtype=np.uint32) if k == "ro" else np.zeros(64, np.uint32))
                for b, k in op.buffers.items()}
        prog, an = check(g["ir"], 1, bufs, [[[k]] for k in range(len(op.instrs))], runtime_flags=rf)
    else:
        txt, size = random_program(1100 + seed, loop=True, n_body=12)
        op = ir.parse(txt)
        grid = 2
        nout = op.nv - 1 + op.ns - 1
        bufs = random_buffers(seed, op.block, grid, size, nout)
        r = np.random.default_rng(seed)
        nw = grid * op.nwarps
        scheds = [[r.integers(0, 60, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)]
                  for _ in range(4)]
        prog, an = check(txt, grid, bufs, scheds, runtime_flags=rf)
    if an.backups:
        assert ("BKS[warp]" if slot == "smem" else "__shfl_sync(0xffffffffu, BKV0") in prog.source
