"""GPU parity for configs[2] (C3 stencil, reverting) and configs[3] (C4a
histogram with OSRB, C4b BFS frontier): small sizes element-by-element
against the oracle interpreter under forced random (nested, poisoned)
preemption; BASELINE sizes under flag preemption at random times against the
uninterrupted run and textbook references (numpy stencil in the IR's f32
order, np.bincount, a plain queue BFS)."""
import time

import numpy as np
import pytest

from oracle import analysis as A
from oracle import interp, ir
from workloads import configs

from gpu_helpers import (check_headers_vs_plans, flag_run, from_dev, gpu_run, header_records,
                         oracle_records, to_dev)

pytestmark = pytest.mark.gpu


def _cb():
    import paper_conf_ipps_jiw21_b200 as cb
    return cb


def forced_parity(cfg, grid, nsched, max_visit, skip=(), compare=None, seed=5, flags=7, prog_flags=0, debug=0):
    cb = _cb()
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT", flags=flags)
    prog = cb.Program(cfg["ir"], flags=flags | prog_flags, poll_policy=cb.POLL_EXPLICIT,
                      debug=cb.DEBUG_FORCED | cb.DEBUG_POISON | debug)
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    names = list(op.buffers)
    uni = cfg["uniforms"]
    ref, _ = interp.run(an, grid, cfg["buffers"], uni)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [None] + [[r.integers(0, max_visit, nw).astype(np.uint32),
                        r.integers(0, max(2, max_visit // 4), nw).astype(np.uint32)] for _ in range(nsched)]
    for sched in scheds:
        s = sched or []
        out, rec = interp.run(an, grid, cfg["buffers"], uni, schedule=s)
        g, hdrs, _ = gpu_run(prog, names, grid, cfg["buffers"], uni, schedule=s)
        for n in names:
            if n in skip:
                continue
            if compare and n in compare:
                compare[n](g[n], out[n], ref[n])
            else:
                assert np.array_equal(g[n], out[n]), n
                assert np.array_equal(out[n], ref[n]), n
        if sched is not None:
            assert header_records(hdrs)[:len(oracle_records(rec, an))] == oracle_records(rec, an)
    return an


def test_c3_small_forced():
    cfg = configs.c3(512, 128, 64)
    an = forced_parity(cfg, 4, 3, 128)
    assert any(an.plans[c].n_revert_res + an.plans[c].n_revert_pre > 0 for c in an.sites)


def test_c3_small_forced_bench_placement():
    """The bench's C3 poll placement (8 rows per iteration, the reverting site
    after the last row's advance only)."""
    cfg = configs.c3(512, 128, 64, **configs.BENCH_C3)
    an = forced_parity(cfg, 4, 3, 16)
    assert len(an.sites) == 1 and an.plans[an.sites[0]].n_revert_res + an.plans[an.sites[0]].n_revert_pre > 0


def test_c3_small_forced_no_spec_restore():
    """The A/B build without speculative restore loads: the
    bench placement's payload is loaded after the header's dispatch."""
    cfg = configs.c3(512, 128, 64, **configs.BENCH_C3)
    forced_parity(cfg, 4, 3, 16, debug=_cb().DEBUG_NO_SPEC_RESTORE)


def test_c3_small_forced_rank_resume():
    """CTXB_RANK_RESUME (NEXT N4) plans on the GPU vs the oracle."""
    cfg = configs.c3(512, 128, 64)
    an = forced_parity(cfg, 4, 3, 128, flags=7 | 32)
    assert all(an.plans[c].p == c for c in an.sites)


@pytest.mark.parametrize("slot", [0, 2048, 4096])   # register, CTXB_OSRB_SMEM, CTXB_OSRB_LANES
def test_c4a_small_forced(slot):
    cfg = configs.c4a(1 << 14, grid=2)
    an = forced_parity(cfg, 2, 3, 4, prog_flags=slot)
    assert an.backups, "C4a must select an OSRB backup"


def test_c4a_small_forced_gather():
    """CTXB_GATHER_RESUME (resumed warps wait until every preempted warp of
    the launch has restored): outputs and headers unchanged, nested."""
    cfg = configs.c4a(1 << 14, grid=2)
    forced_parity(cfg, 2, 3, 4, flags=7 | 128)


def test_c3_small_forced_gather():
    cfg = configs.c3(512, 128, 64)
    forced_parity(cfg, 4, 3, 128, flags=7 | 128)


@pytest.mark.parametrize("flags,polls", [(7, "both"), (7 | 32, "both"), (7, configs.BENCH_C4B_POLLS)])
def test_c4b_small_forced_level(flags, polls):
    rp, ci = configs.c4b_graph(1 << 10, 16)
    n = len(rp) - 1
    dist = np.full(n, 0xFFFFFFFF, np.uint32)
    dist[0] = 0
    # level 1 frontier = neighbours of 0 already discovered: run level 0 and 1 kernels
    front = np.array([0], np.uint32)
    for lvl in range(3):
        cfg = dict(ir=configs.c4b_ir(polls), uniforms={"nf": len(front), "lvl1": lvl + 1},
                   buffers={"rowptr": rp, "colidx": ci, "front": np.pad(front, (0, 1)),
                            "dist": dist.copy(), "nextf": np.zeros(n, np.uint32),
                            "nextcnt": np.zeros(1, np.uint32)})

        def cmp_nextf(g, o, ref, cnt=None):
            pass
        forced_parity(cfg, 2, 2, 40, skip=("nextf",), flags=flags)
        # advance with the oracle (frontier order is irrelevant to the next level's dist)
        op = ir.parse(cfg["ir"])
        an = A.analyze(op, policy="EXPLICIT")
        out, _ = interp.run(an, 2, cfg["buffers"], cfg["uniforms"])
        cnt = int(out["nextcnt"][0])
        front = np.sort(out["nextf"][:cnt])
        dist = out["dist"]
        if cnt == 0:
            break


def _persistent_grid(prog):
    bps, nsm = prog.occupancy()
    return bps * nsm


@pytest.mark.parametrize("flags,variant", [(7, {}), (7 | 32, {}), (7, configs.BENCH_C3)])
def test_c3_full_flag(flags, variant):
    import torch
    cb = _cb()
    cfg = configs.c3(**variant)
    W, H = cfg["W"], cfg["H"]
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT", flags=flags)
    prog = cb.Program(cfg["ir"], flags=flags, poll_policy=cb.POLL_EXPLICIT)
    grid = _persistent_grid(prog)
    dX = to_dev(cfg["buffers"]["X"])
    dY = torch.zeros(W * H, dtype=torch.int32, device="cuda")
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    run = prog.launch(grid, [dX, dY], [], ctx, s)
    assert run.wait()
    T = run.launch_ms() / 1e3
    ref = dY.clone()
    assert np.array_equal(from_dev(ref), configs.c3_numpy_reference(cfg["buffers"]["X"], W, H))
    sb = [an.plans[c].payload_bytes for c in an.sites]
    lb = [an.live[c].payload_bytes for c in an.sites]
    npre = 0
    for fr in (0.2, 0.5, 0.8):
        dY.zero_()
        torch.cuda.synchronize()
        st, hdr, _ = flag_run(prog, grid, [dX, dY], [], ctx, fr * T, s, ctrl)
        torch.cuda.synchronize()
        npre += st["warps_preempted"]
        check_headers_vs_plans(hdr, 1, sb, lb)
        assert torch.equal(dY, ref)
    assert npre > 0


@pytest.mark.parametrize("skewed,gather", [(False, 0), (True, 0), (False, 128), (True, 256), (False, 384)])
def test_c4a_full_flag(skewed, gather):
    import torch
    cb = _cb()
    cfg = configs.c4a(1 << 28, skewed=skewed, grid=1)
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | gather)
    assert prog.backups == an.backups and prog.backups
    grid = _persistent_grid(prog)
    keys = cfg["buffers"]["keys"]
    want = np.bincount(keys >> 24, minlength=256).astype(np.uint32)
    dK, dS = to_dev(keys), to_dev(cfg["buffers"]["starts"])
    dH = torch.zeros(256 * grid, dtype=torch.int32, device="cuda")
    total = lambda: from_dev(dH).reshape(grid, 256).astype(np.uint64).sum(0).astype(np.uint32)  # noqa: E731
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    run = prog.launch(grid, [dK, dS, dH], [], ctx, s)
    assert run.wait()
    T = run.launch_ms() / 1e3
    assert np.array_equal(total(), want)
    sb = [an.plans[c].payload_bytes for c in an.sites]
    lb = [an.live[c].payload_bytes for c in an.sites]
    for fr in (0.3, 0.7):
        dH.zero_()
        torch.cuda.synchronize()
        st, hdr, _ = flag_run(prog, grid, [dK, dS, dH], [], ctx, fr * T, s, ctrl)
        torch.cuda.synchronize()
        check_headers_vs_plans(hdr, 1, sb, lb)
        assert np.array_equal(total(), want)


@pytest.mark.parametrize("replicas,polls", [(False, "both"), (True, "both"), (True, configs.BENCH_C4B_POLLS)])
def test_c4b_full_flag(replicas, polls):
    import torch
    cb = _cb()
    rp, ci = configs.c4b_graph()
    n = len(rp) - 1
    want = configs.bfs_reference(rp, ci)
    op = ir.parse(configs.c4b_ir(polls))
    an = A.analyze(op, policy="EXPLICIT")
    prog = cb.Program(configs.c4b_ir(polls), poll_policy=cb.POLL_EXPLICIT,
                      flags=cb.ALL | (cb.FLAG_REPLICAS if replicas else 0))
    grid = _persistent_grid(prog)
    sb = [an.plans[c].payload_bytes for c in an.sites]
    lb = [an.live[c].payload_bytes for c in an.sites]
    d_rp, d_ci = to_dev(rp), to_dev(ci)
    dist = np.full(n, 0xFFFFFFFF, np.uint32)
    dist[0] = 0
    d_dist = to_dev(dist)
    fronts = [to_dev(np.zeros(n + 1, np.uint32)), to_dev(np.zeros(n + 1, np.uint32))]
    fronts[0][0] = 0
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    nf, lvl, npre = 1, 0, 0
    r = np.random.default_rng(300)
    while nf:
        cnt.zero_()
        torch.cuda.synchronize()
        bufs = [d_rp, d_ci, fronts[lvl % 2], d_dist, fronts[(lvl + 1) % 2], cnt]
        st, hdr, _ = flag_run(prog, grid, bufs, [nf, lvl + 1], ctx, float(r.uniform(0, 2e-4)), s, ctrl)
        torch.cuda.synchronize()
        npre += st["warps_preempted"]
        check_headers_vs_plans(hdr, 1, sb, lb)
        newf = np.sort(from_dev(fronts[(lvl + 1) % 2])[:int(cnt.item())])
        wantf = np.sort(np.nonzero(want == lvl + 1)[0].astype(np.uint32))
        assert np.array_equal(newf, wantf), f"level {lvl + 1} frontier differs (as a multiset)"
        nf = int(cnt.item())
        lvl += 1
    assert np.array_equal(from_dev(d_dist), want)


@pytest.mark.parametrize("grid_kind", ["persistent", "occupancy"])
def test_c4a_library_defaults(grid_kind):
    """The library's defaults on C4a: watcher + drain notice +
    synchronous test, gathered resume (atomics).  preempt(None) signals through
    the watcher alone.  On the occupancy grid one block cannot be resident
    beside the watcher, so the resume must not gather (it would wait for that
    block); on the persistent grid it gathers.  Bit-exact either way."""
    import torch
    cb = _cb()
    cfg = configs.c4a(1 << 26, grid=1)
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT)
    want_bits = cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL | cb.GATHER_RESUME
    assert prog.info["flags"] & want_bits == want_bits
    grid = prog.persistent_grid() if grid_kind == "persistent" else _persistent_grid(prog)
    keys = cfg["buffers"]["keys"]
    want = np.bincount(keys >> 24, minlength=256).astype(np.uint32)
    dK, dS = to_dev(keys), to_dev(cfg["buffers"]["starts"])
    dH = torch.zeros(256 * grid, dtype=torch.int32, device="cuda")
    total = lambda: from_dev(dH).reshape(grid, 256).astype(np.uint64).sum(0).astype(np.uint32)  # noqa: E731
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    run = prog.launch(grid, [dK, dS, dH], [], ctx, s)
    assert run.wait()
    T = run.launch_ms() / 1e3
    assert np.array_equal(total(), want)
    preempted = 0
    for fr in (0.2, 0.5, 0.8):
        dH.zero_()
        torch.cuda.synchronize()
        st, _, _ = flag_run(prog, grid, [dK, dS, dH], [], ctx, fr * T, s, None)
        torch.cuda.synchronize()
        preempted += st["warps_preempted"]
        assert np.array_equal(total(), want), fr
    assert preempted > 0
