"""GPU parity on the BASELINE.json configs beyond C1 (C2 tiled SGEMM), and the
bulk save/restore microbench's correctness.

* C2 at a small size: the generated kernel's C equals the oracle interpreter's
  bit for bit, uninterrupted and under forced random per-warp preemption
  (nested, poisoned), with per-warp context bytes equal to the oracle's;
* C2 at the full BASELINE size (4096^3, 148 SMs x occupancy persistent grid):
  sampled C elements equal the oracle's correctly rounded f32 fma chain in the
  IR's k order; preemption by the flag at random times + resume gives C
  bit-exact with the uninterrupted run; every preempted warp's header bytes
  equal the oracle plan's bytes for the site it reports.
"""
import numpy as np
import pytest

from oracle import analysis as A
from oracle import fp32, interp, ir
from workloads import configs

from gpu_helpers import from_dev, gpu_run, header_records, oracle_records, to_dev

pytestmark = pytest.mark.gpu


def _cb():
    import paper_conf_ipps_jiw21_b200 as cb
    return cb


@pytest.mark.parametrize("size,grid,nsched,polls", [((128, 128, 64), 1, 3, "iter"), ((128, 128, 32), 1, 3, "half"),
                                                    ((256, 256, 32), 4, 1, "iter")])
def test_c2_small_forced(size, grid, nsched, polls):
    cb = _cb()
    M, N, K = size
    cfg = configs.c2(M, N, K, polls=polls)
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_FORCED | cb.DEBUG_POISON,
                      min_blocks_per_sm=cfg["min_blocks"])
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    names = list(op.buffers)
    ref, _ = interp.run(an, grid, cfg["buffers"])
    g0, _h, _ = gpu_run(prog, names, grid, cfg["buffers"], {})
    assert np.array_equal(g0["C"], ref["C"])
    per_iter = {"iter": 1, "step": 4, "half": 8}[polls]
    visits = (K // 4) * per_iter * (M * N // (128 * 128) // grid)
    r = np.random.default_rng(5)
    nw = grid * 8
    for _ in range(nsched):
        sched = [r.integers(0, visits, nw).astype(np.uint32), r.integers(0, 40, nw).astype(np.uint32)]
        out, rec = interp.run(an, grid, cfg["buffers"], schedule=sched)
        assert np.array_equal(out["C"], ref["C"])
        g, hdrs, _ = gpu_run(prog, names, grid, cfg["buffers"], {}, schedule=sched)
        assert np.array_equal(g["C"], ref["C"])
        assert header_records(hdrs)[:len(oracle_records(rec, an))] == oracle_records(rec, an)


def test_c2_full_size_flag_preemption():
    import time
    import torch
    cb = _cb()
    cfg = configs.c2()
    M, N, K = cfg["M"], cfg["N"], cfg["K"]
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=cfg["min_blocks"])
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    bps, nsm = prog.occupancy()
    assert bps == 2
    grid = bps * nsm
    dA, dB = to_dev(cfg["buffers"]["A"]), to_dev(cfg["buffers"]["B"])
    dC = torch.zeros(M * N, dtype=torch.int32, device="cuda")
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    ctrl = torch.cuda.Stream()
    t0 = time.time()
    run = prog.launch(grid, [dA, dB, dC], [], ctx, s)
    assert run.wait()
    t_unint = time.time() - t0
    ref = dC.clone()
    # sampled elements vs the oracle's f32 fma chain in the IR's k order
    rng = np.random.default_rng(17)
    rows = rng.integers(0, M, 256)
    cols = rng.integers(0, N, 256)
    A_ = cfg["buffers"]["A"]
    B_ = cfg["buffers"]["B"]
    acc = np.zeros(256, dtype=np.uint32)
    for k in range(K):
        acc = fp32.ffma(A_[rows * K + k], B_[k * N + cols], acc)
    got = from_dev(ref)[rows * N + cols]
    assert np.array_equal(got, acc)
    site_bytes = {k: an.plans[c].payload_bytes for k, c in enumerate(an.sites)}
    live_bytes = {k: an.live[c].payload_bytes for k, c in enumerate(an.sites)}
    for trial in range(3):
        dC.zero_()
        torch.cuda.synchronize()
        run = prog.launch(grid, [dA, dB, dC], [], ctx, s)
        time.sleep(t_unint * (0.1 + 0.3 * trial))
        st = run.preempt(ctrl)
        if st["warps_preempted"]:
            h = run.headers()
            for w in range(h.shape[0]):
                if h[w, 2] == 1 and h[w, 3] == 1:
                    k, live = int(h[w, 0]) & 0x7FFFFFFF, bool(h[w, 0] >> 31)
                    assert int(h[w, 1]) == (live_bytes[k] if live else site_bytes[k])
            assert st["payload_bytes"] == run.context_bytes()[0]
            run.resume(s)
            assert run.wait()
        torch.cuda.synchronize()
        assert torch.equal(dC, ref), f"trial {trial}: C after preempt/resume differs"


def test_bulk_save_restore_roundtrip():
    import torch
    cb = _cb()
    prog = cb.Program(configs.bulk_ir(64), poll_policy=cb.POLL_EXPLICIT, mode=cb.MODE_LIVE,
                      debug=cb.DEBUG_FORCED, min_blocks_per_sm=configs.BULK_MIN_BLOCKS)
    grid = 2048
    nw = grid * 8
    out = torch.zeros(256, dtype=torch.int32, device="cuda")
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    run = prog.launch(grid, [out], [], ctx, forced=np.zeros(nw, np.uint32))
    assert not run.wait()
    h = run.headers()
    assert (h[:, 2] == 1).all() and (h[:, 1] == 64 * 128).all()
    # payload of warp w: group g lane l holds values 4g..4g+3 of thread 32*(w%8)+l
    pay_off = ((nw * 16 + 255) // 256) * 256
    raw = ctx[pay_off:pay_off + 8 * 8192].cpu().numpy().view(np.uint32).reshape(8, 16, 32, 4)
    tid = (np.arange(8)[:, None] * 32 + np.arange(32)[None, :]).astype(np.uint32)
    for g in range(16):
        for q in range(4):
            i = 4 * g + q
            want = tid ^ np.uint32(((i + 1) * 0x9E3779B9) & 0xFFFFFFFF)
            assert np.array_equal(raw[:, g, :, q], want)
    run.resume(forced=np.full(nw, cb.NEVER, np.uint32))
    assert run.wait()
    assert int(out.abs().sum()) == 0


def test_c2s_smem_small_forced_block_uniform():
    """NEXT N2: shared memory + barriers.  Preemption is block-uniform at the
    barriers (any warp's decision preempts the block); each warp saves its
    register plan and a slice of the block's shared memory; both are
    poisoned and restored.  GPU == oracle, headers == oracle records."""
    cb = _cb()
    cfg = configs.c2s(128, 128, 32)
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_FORCED | cb.DEBUG_POISON,
                      min_blocks_per_sm=2)
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    names = list(op.buffers)
    ref, _ = interp.run(an, 1, cfg["buffers"])
    g0, _h, _ = gpu_run(prog, names, 1, cfg["buffers"], {})
    assert np.array_equal(g0["C"], ref["C"])
    r = np.random.default_rng(8)
    for _ in range(4):
        sched = [r.integers(0, 8, 8).astype(np.uint32), r.integers(0, 4, 8).astype(np.uint32)]
        out, rec = interp.run(an, 1, cfg["buffers"], schedule=sched)
        assert np.array_equal(out["C"], ref["C"])
        g, hdrs, _ = gpu_run(prog, names, 1, cfg["buffers"], {}, schedule=sched)
        assert np.array_equal(g["C"], ref["C"])
        orc = oracle_records(rec, an)
        assert header_records(hdrs)[:len(orc)] == orc
        for launch in orc:                      # block-uniform: all 8 warps of the block together
            assert len(launch) in (0, 8)


def test_c2s_full_flag_equals_c2():
    import time
    import torch
    cb = _cb()
    cfg = configs.c2s()
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)
    c2p = cb.Program(configs.c2()["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)
    bps, nsm = prog.occupancy()
    grid = min(bps, c2p.occupancy()[0]) * nsm
    dA, dB = to_dev(cfg["buffers"]["A"]), to_dev(cfg["buffers"]["B"])
    dC = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    ctx2 = torch.zeros(c2p.context_capacity(grid), dtype=torch.uint8, device="cuda")
    r2 = c2p.launch(grid, [dA, dB, dC], [], ctx2, s)
    assert r2.wait()
    ref = dC.clone()
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    dC.zero_()
    run = prog.launch(grid, [dA, dB, dC], [], ctx, s)
    assert run.wait()
    T = run.launch_ms() / 1e3
    assert torch.equal(dC, ref), "C2s (shared-memory tiles) must equal C2 bit for bit"
    npre = 0
    for fr in (0.2, 0.5, 0.8):
        dC.zero_()
        torch.cuda.synchronize()
        run = prog.launch(grid, [dA, dB, dC], [], ctx, s)
        t0 = time.perf_counter()
        while time.perf_counter() < t0 + fr * T:
            pass
        st = run.preempt(ctrl)
        npre += st["warps_preempted"]
        if st["warps_preempted"]:
            h = run.headers()
            pre = (h[:, 2] == 1) & (h[:, 3] == 1)
            assert pre.reshape(-1, 8).all(axis=1).sum() == st["blocks_preempted"]   # whole blocks
            run.resume(s)
            assert run.wait()
        torch.cuda.synchronize()
        assert torch.equal(dC, ref)
    assert npre > 0


@pytest.mark.parametrize("which,host", [("c2", False), ("c3", False), ("c2s", False),
                                        ("c2", True), ("c3", True), ("c2s", True),
                                        ("c2", "armed"), ("c3", "armed"),
                                        ("c3", "replicas"), ("c2", "replicas"), ("c3", "load4"),
                                        ("c3", "replicas+load4"), ("c3r2", "load4"),
                                        ("c3r2", "combo"), ("c2", "combo"), ("c4a", "combo"), ("c4a", False),
                                        ("c2", "notice"), ("c3r2", "notice"), ("c2s", "notice"),
                                        ("c2", "watcher"), ("c3b", "watcher"), ("c4a", "watcher"), ("c2s", "watcher"),
                                        ("c2", "watcher_only"), ("c3b", "watcher_only"), ("c2", "watcher_gather"),
                                        ("c3b", "watcher_gather"), ("c2", "watcher_noctrl"), ("c4a", "watcher_noctrl"),
                                        ("c2", "watcher_sync"), ("c3b", "watcher_sync"), ("c2s", "watcher_sync")])
def test_flag_mode_repeated_nested_preemption(which, host, monkeypatch):
    """random flag times, repeated and nested
    preempt -> resume -> preempt ... cycles (each resume can be preempted
    again, also inside the same basic-block pass: the LIVE fallback, R-16);
    the final output stays bit-exact with the uninterrupted run.  host=True:
    CTXB_HOST_SIGNAL with the stream-memop fallback disabled
    (CTXB_HOST_SIGNAL_ONLY=1), so every preemption arrives through a relay
    warp's system-scope poll of the host word.  host="armed":
    CTXB_ARMED_SIGNAL, every launch and resume pre-enqueues its signal behind
    a host gate; runs that end unpreempted are disarmed.
    "replicas" / "load4": CTXB_FLAG_REPLICAS (master pollers forward the
    signal to 64 replicas) and loads at every 4th poll visit.
    "watcher": CTXB_WATCHER (+ drain notice) -- a co-resident warp relays the
    host store; "watcher_only": without the memop fallback, so
    every preemption arrives through the watcher."""
    import time
    import torch
    cb = _cb()
    if which == "c4a":
        cfg = configs.c4a(1 << 28, grid=1)
        bufs = [to_dev(cfg["buffers"]["keys"]), to_dev(cfg["buffers"]["starts"]), None]
        out_i, mb = 2, 0
    elif which in ("c3", "c3r2", "c3b"):
        cfg = configs.c3(**configs.BENCH_C3) if which == "c3b" else configs.c3(rows_per_iter=2 if which == "c3r2" else 1)
        bufs = [to_dev(cfg["buffers"]["X"]), torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")]
        out_i, mb = 1, 0
    else:
        cfg = configs.c2() if which == "c2" else configs.c2s()
        bufs = [to_dev(cfg["buffers"]["A"]), to_dev(cfg["buffers"]["B"]),
                torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")]
        out_i, mb = 2, 2
    if host is True or host == "watcher_only":
        monkeypatch.setenv("CTXB_HOST_SIGNAL_ONLY", "1")
    # "combo": the runtime options together (armed signal, gathered resume, flag
    # replicas, sparse flag loads; C4a also the synchronous test and shared-memory OSRB slots)
    combo = cb.ARMED_SIGNAL | cb.GATHER_RESUME | cb.FLAG_REPLICAS | cb.DRAIN_NOTICE
    if which == "c4a":
        combo |= cb.SYNC_POLL | cb.OSRB_SMEM
    extra = {"armed": cb.ARMED_SIGNAL, "replicas": cb.FLAG_REPLICAS, "load4": 0, "combo": combo,
             "notice": cb.DRAIN_NOTICE | cb.ARMED_SIGNAL,
             "watcher": cb.WATCHER | cb.DRAIN_NOTICE, "watcher_only": cb.WATCHER,
             "watcher_gather": cb.WATCHER | cb.DRAIN_NOTICE | cb.GATHER_RESUME,
             "watcher_noctrl": cb.WATCHER | cb.DRAIN_NOTICE,
             "watcher_sync": cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL,   # the bench's signal path
             "replicas+load4": cb.FLAG_REPLICAS, True: cb.HOST_SIGNAL, False: 0}[host]
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=mb, flags=cb.ALL | extra,
                      load_every=4 if host in ("load4", "replicas+load4", "combo") else 1)
    grid = prog.persistent_grid()
    if host in ("watcher", "watcher_only", "watcher_gather", "watcher_noctrl", "watcher_sync") and which in ("c2", "c2s"):
        bps, nsm = prog.occupancy()
        assert grid == bps * nsm - 1      # the full register file leaves no room for the watcher warp
    if bufs[out_i] is None:
        bufs[out_i] = torch.zeros(256 * grid, dtype=torch.int32, device="cuda")
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    if host == "watcher_noctrl":   # the watcher alone: no control stream, no memop fallback
        ctrl = None
    run = prog.launch(grid, bufs, [], ctx, s)
    assert run.wait()
    T = run.launch_ms() / 1e3
    ref = bufs[out_i].clone()
    rng = np.random.default_rng(77)
    total_pre = cycles = 0
    for trial in range(3):
        bufs[out_i].zero_()
        torch.cuda.synchronize()
        run = prog.launch(grid, bufs, [], ctx, s)
        while True:
            t0 = time.perf_counter()
            while time.perf_counter() < t0 + rng.uniform(0.02, 0.25) * T:
                pass
            st = run.preempt(ctrl)
            if not st["warps_preempted"]:
                break
            total_pre += st["warps_preempted"]
            cycles += 1
            run.resume(s)
            if cycles > 40:
                assert run.wait() or True
                break
        if not run.wait():
            while not run.finished:
                run.resume(s)
                run.wait()
        torch.cuda.synchronize()
        assert torch.equal(bufs[out_i], ref), f"{which}: output differs after {cycles} nested cycles"
    assert cycles >= 3 and total_pre > 0


@pytest.mark.parametrize("armed,use_async", [(False, False), (True, False), (False, True), (True, True)])
def test_statless_preempt_settles_lazily(armed, use_async):
    """ctxb_preempt with NULL stats returns once drained (state settled on the
    next call): repeated nested cycles on C3 with stats=False stay bit-exact,
    drain_stats() matches the header counts, and a finished run reports done."""
    import time
    import torch
    cb = _cb()
    cfg = configs.c3()
    bufs = [to_dev(cfg["buffers"]["X"]), torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")]
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | (cb.ARMED_SIGNAL if armed else 0))
    bps, nsm = prog.occupancy()
    grid = bps * nsm
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    run = prog.launch(grid, bufs, [], ctx, s)
    assert run.wait()
    T = run.launch_ms() / 1e3
    ref = bufs[1].clone()
    rng = np.random.default_rng(5)
    npre = 0
    for trial in range(4):
        bufs[1].zero_()
        torch.cuda.synchronize()
        run = prog.launch(grid, bufs, [], ctx, s)
        for _ in range(6):
            t0 = time.perf_counter()
            while time.perf_counter() < t0 + rng.uniform(0.05, 0.3) * T:
                pass
            if use_async:   # ctxb_preempt_async: returns at once, wait() observes the drain
                run.preempt_async(ctrl)
                run.wait()
            else:
                assert run.preempt(ctrl, stats=False) is None
            if run.finished:
                break
            d = run.drain_stats()
            h = run.headers()
            assert d["warps_preempted"] == int((h[:, 2] == 1).sum()) > 0
            assert d["payload_bytes"] == int(h[h[:, 2] == 1, 1].astype(np.int64).sum())
            npre += d["warps_preempted"]
            run.resume(s)
        while not run.wait():
            run.resume(s)
        torch.cuda.synchronize()
        assert torch.equal(bufs[1], ref)
    assert npre > 0


def test_destroy_running_armed_run_completes():
    """Dropping a run handle while its (armed) launch runs waits for the launch
    instead of firing the armed signal into it: the output is complete, and the
    pooled resources serve the next run, which preempts and resumes bit-exact."""
    import torch
    cb = _cb()
    cfg = configs.c3()
    X = to_dev(cfg["buffers"]["X"])
    Y = torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | cb.ARMED_SIGNAL)
    bps, nsm = prog.occupancy()
    grid = bps * nsm
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    run = prog.launch(grid, [X, Y], [], ctx, s)
    assert run.wait()
    ref = Y.clone()
    Y.zero_()
    torch.cuda.synchronize()
    run = prog.launch(grid, [X, Y], [], ctx, s)
    del run                                    # still running: destroy waits, no preemption
    torch.cuda.synchronize()
    assert torch.equal(Y, ref)
    Y.zero_()
    torch.cuda.synchronize()
    run = prog.launch(grid, [X, Y], [], ctx, s)
    st = run.preempt(ctrl)
    if st["warps_preempted"]:
        run.resume(s)
    assert run.wait()
    torch.cuda.synchronize()
    assert torch.equal(Y, ref)


def test_preempt_timeout_leaves_run_running(monkeypatch):
    """CTXB_PREEMPT_TIMEOUT_US: a kernel whose poll sites are compiled out
    cannot drain; ctxb_preempt gives up with CTXB_E_TIMEOUT, the run keeps
    running, ctxb_wait then sees it finish, and the output is complete.  With
    a generous timeout a normal kernel preempts and resumes bit-exact."""
    import torch
    cb = _cb()
    cfg = configs.c3()
    X = to_dev(cfg["buffers"]["X"])
    Y = torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")
    s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
    nopoll = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_POLLS)
    grid = nopoll.occupancy()[0] * nopoll.occupancy()[1]
    ctx = torch.zeros(nopoll.context_capacity(grid), dtype=torch.uint8, device="cuda")
    run = nopoll.launch(grid, [X, Y], [], ctx, s)
    assert run.wait()
    ref = Y.clone()
    Y.zero_()
    torch.cuda.synchronize()
    monkeypatch.setenv("CTXB_PREEMPT_TIMEOUT_US", "50")
    run = nopoll.launch(grid, [X, Y], [], ctx, s)
    with pytest.raises(cb.CtxbError) as ei:
        run.preempt(ctrl)
    assert ei.value.code == cb.E_TIMEOUT
    assert run.wait()                      # it ran to completion
    torch.cuda.synchronize()
    assert torch.equal(Y, ref)
    monkeypatch.setenv("CTXB_PREEMPT_TIMEOUT_US", "1000000")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT)
    ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    Y.zero_()
    torch.cuda.synchronize()
    run = prog.launch(grid, [X, Y], [], ctx, s)
    st = run.preempt(ctrl)
    if st["warps_preempted"]:
        run.resume(s)
    assert run.wait()
    torch.cuda.synchronize()
    assert torch.equal(Y, ref)


def test_program_destroyed_before_its_run():
    """ctxb_program_destroy while a run still references the program defers
    the free to the last run's destruction (any finalisation order is safe)."""
    import gc
    import torch
    cb = _cb()
    cfg = configs.c3(512, 128, 64)
    X = to_dev(cfg["buffers"]["X"])
    Y = torch.zeros(512 * 128, dtype=torch.int32, device="cuda")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT)
    ctx = torch.zeros(prog.context_capacity(4), dtype=torch.uint8, device="cuda")
    run = prog.launch(4, [X, Y], [], ctx)
    assert cb.lib.ctxb_program_destroy(prog._h) == 0   # the run still holds it
    prog._h = None
    assert run.wait()
    del run, prog
    gc.collect()
    torch.cuda.synchronize()
    p2 = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT)   # the library is still healthy
    r2 = p2.launch(4, [X, Y], [], ctx)
    assert r2.wait()


def test_two_runs_with_watchers_concurrently():
    """Two programs, each launch with its own watcher warp, running at the
    same time on two streams (small grids, so both are resident): preempt
    both through their watchers alone, resume both, outputs bit-exact; then
    the same without preemption (each wait releases its watcher)."""
    import time
    import torch
    cb = _cb()
    c3 = configs.c3(2048, 2048, 64, **configs.BENCH_C3)
    x = to_dev(c3["buffers"]["X"])
    y = torch.zeros(2048 * 2048, dtype=torch.int32, device="cuda")
    c2 = configs.c2(1024, 1024, 1024)
    a, b = to_dev(c2["buffers"]["A"]), to_dev(c2["buffers"]["B"])
    c = torch.zeros(1024 * 1024, dtype=torch.int32, device="cuda")
    fl = cb.ALL | cb.WATCHER | cb.DRAIN_NOTICE
    p3 = cb.Program(c3["ir"], poll_policy=cb.POLL_EXPLICIT, flags=fl)
    p2 = cb.Program(c2["ir"], poll_policy=cb.POLL_EXPLICIT, flags=fl, min_blocks_per_sm=2)
    g3, g2 = 32, 16
    ctx3 = torch.zeros(p3.context_capacity(g3), dtype=torch.uint8, device="cuda")
    ctx2 = torch.zeros(p2.context_capacity(g2), dtype=torch.uint8, device="cuda")
    s3, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    r3, r2 = p3.launch(g3, [x, y], [], ctx3, s3), p2.launch(g2, [a, b, c], [], ctx2, s2)
    assert r3.wait() and r2.wait()
    ref3, ref2 = y.clone(), c.clone()
    npre = 0
    for delay in (20e-6, 200e-6):
        y.zero_()
        c.zero_()
        torch.cuda.synchronize()
        r3, r2 = p3.launch(g3, [x, y], [], ctx3, s3), p2.launch(g2, [a, b, c], [], ctx2, s2)
        t0 = time.perf_counter()
        while time.perf_counter() < t0 + delay:
            pass
        st3, st2 = r3.preempt(None), r2.preempt(None)
        npre += st3["warps_preempted"] + st2["warps_preempted"]
        for r, s in ((r3, s3), (r2, s2)):
            while not r.finished:
                r.resume(s)
                r.wait()
        torch.cuda.synchronize()
        assert torch.equal(y, ref3) and torch.equal(c, ref2)
    assert npre > 0


@pytest.mark.parametrize("which,path", [("c3", "watcher"), ("c2", "watcher"), ("c3", "armed"), ("c3", "memop")])
def test_watcher_lifecycle_fuzz(which, path):
    """Seeded random sequences of the run API on the watcher path (C3, C2) and
    the armed path (C3):
    preempt with and without stats, preempt_async, blocking waits on
    unpreempted launches, query polling, resumes, and runs dropped while
    still running; every job's output bit-exact and nothing hangs (a
    watchdog aborts the process instead of letting a deadlock sit)."""
    import faulthandler
    import sys
    import time
    import torch
    cb = _cb()
    faulthandler.dump_traceback_later(240, exit=True, file=sys.stderr)
    try:
        fl = {"watcher": cb.WATCHER | cb.DRAIN_NOTICE | cb.SYNC_POLL, "armed": cb.ARMED_SIGNAL, "memop": 0}[path]
        if which == "c3":
            cfg = configs.c3(**configs.BENCH_C3)
            ins = [to_dev(cfg["buffers"]["X"])]
            y = torch.zeros(cfg["W"] * cfg["H"], dtype=torch.int32, device="cuda")
            mb = 0
        else:
            cfg = configs.c2()
            ins = [to_dev(cfg["buffers"]["A"]), to_dev(cfg["buffers"]["B"])]
            y = torch.zeros(cfg["M"] * cfg["N"], dtype=torch.int32, device="cuda")
            mb = 2
        prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | fl, min_blocks_per_sm=mb)
        grid = prog.persistent_grid()
        ctx = torch.zeros(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        s, ctrl = torch.cuda.Stream(), torch.cuda.Stream()
        bufs = ins + [y]
        run = prog.launch(grid, bufs, [], ctx, s)
        assert run.wait()
        T = run.launch_ms() / 1e3
        ref = y.clone()
        import os
        rng = np.random.default_rng(int(os.environ.get("CTXB_FUZZ_SEED", "2024")))
        npre = 0
        for job in range(int(os.environ.get("CTXB_FUZZ_JOBS", "40"))):
            y.zero_()
            torch.cuda.synchronize()
            run = prog.launch(grid, bufs, [], ctx, s)
            op = int(rng.integers(6))
            t0 = time.perf_counter()
            while time.perf_counter() < t0 + rng.uniform(0.0, 0.9) * T:
                pass
            if op == 5:                       # drop the run while it may still run; the destructor waits
                del run
                torch.cuda.synchronize()
                assert torch.equal(y, ref)
                continue
            c0 = None if path == "watcher" and rng.integers(2) else ctrl   # armed: ctrl unused
            if op == 0:
                st = run.preempt(c0)
                npre += st["warps_preempted"]
            elif op == 1:
                assert run.preempt(c0, stats=False) is None
            elif op == 2:
                run.preempt_async(c0)
            elif op == 3:
                while run.running():
                    pass
            # op 4: no preemption, a blocking wait
            while not run.wait():
                if rng.integers(3) == 0:      # preempt the resumed launch again at once
                    run.resume(s)
                    st = run.preempt(ctrl)
                    npre += st["warps_preempted"]
                    continue
                run.resume(s)
            torch.cuda.synchronize()
            assert torch.equal(y, ref), f"job {job} (op {op}) differs"
        assert npre > 0
    finally:
        faulthandler.cancel_dump_traceback_later()


def test_c2_resumed_kernel_runs_at_normal_speed():
    """C2 preempted at every warp's first poll visit (forced), so
    the resume kernel does almost all of the work: bit-exact, and it takes no
    more than 1.10x the uninterrupted kernel (measured 1.01x; before the resume code re-entered
    loops through a peeled copy and recomputed the lane offsets: 3x)."""
    import torch
    cb = _cb()
    cfg = configs.c2()
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_FORCED, min_blocks_per_sm=2)
    grid = prog.persistent_grid()
    nw = grid * 8
    dA, dB = (torch.from_numpy(cfg["buffers"][n].view(np.int32)).cuda() for n in ("A", "B"))
    dC = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    never = np.full(nw, cb.NEVER, np.uint32)
    ts = []
    for _ in range(3):
        run = prog.launch(grid, [dA, dB, dC], [], ctx, forced=never)
        assert run.wait()
        ts.append(run.launch_ms())
    ref = dC.clone()
    dC.zero_()
    run = prog.launch(grid, [dA, dB, dC], [], ctx, forced=np.full(nw, 1, np.uint32))
    assert not run.wait()
    run.resume(forced=never)
    assert run.wait()
    t_res = run.launch_ms()
    torch.cuda.synchronize()
    assert torch.equal(dC, ref)
    assert t_res < 1.10 * float(np.median(ts)), (t_res, ts)
