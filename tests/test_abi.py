"""CPU tests of the C-ABI library: it loads without a GPU, exports every
symbol include/ctxb.h declares, reports errors through status codes, and its
analyzer (C++, independent of the oracle) produces plans identical to the
oracle's on random programs and the configs (parity of the compile-time
part, runs without a GPU)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import ir
from workloads import configs
from workloads.randprog import random_program

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "ctxb.h")).read()
    return sorted(set(re.findall(r"\b(ctxb_[a-z_]+)\s*\(", txt)))


def test_library_exports_every_header_symbol():
    lib = ctypes.CDLL(cb.LIB_PATH)
    syms = header_symbols()
    assert len(syms) >= 19
    for s in syms:
        assert hasattr(lib, s), s
    assert sorted(cb.EXPORTED_SYMBOLS) == syms


def test_parse_errors_are_status_codes():
    bad = [".kernel k\n.vregs 1\n.sregs 0\n.block 32\n  bogus v0\n  exit\n",
           ".kernel k\n.vregs 1\n.sregs 0\n.block 33\n  exit\n",
           ".kernel k\n.vregs 1\n.sregs 1\n.block 32\n  mov s0, %tid\n  exit\n",
           ".kernel k\n.vregs 1\n.sregs 0\n.block 32\n  mov v3, 1\n  exit\n",
           ".kernel k\n.vregs 1\n.sregs 0\n.block 32\n  mov v0, 1\n"]
    for t in bad:
        with pytest.raises(cb.CtxbError) as e:
            cb.Program(t, debug=cb.DEBUG_NO_COMPILE)
        assert e.value.code == -2
        with pytest.raises(ir.IRError):
            ir.parse(t)


def test_gpu_calls_fail_loudly_without_device():
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("a GPU is present")
    except Exception:
        pass
    p = cb.Program(configs.c1()["ir"], debug=cb.DEBUG_NO_COMPILE)
    with pytest.raises(cb.CtxbError):
        p.launch(1, [1, 2, 3, 4], [], 5, ctx_bytes=1 << 20)


def _same_plans(txt, policy="EVERY_INSTR", flags=7, mode=0):
    op = ir.parse(txt)
    an = A.analyze(op, policy=policy, flags=flags, mode=mode)
    pol = {"EVERY_INSTR": 0, "EVERY_N": 1, "EXPLICIT": 2}[policy]
    p = cb.Program(txt, flags=flags, mode=mode, poll_policy=pol, debug=cb.DEBUG_NO_COMPILE)
    assert p.num_sites == len(an.sites)
    assert p.backups == an.backups
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c]), (k, c)
        assert p.plan_text(k, live=True) == A.plan_text(op, an.live[c])
        si = p.site_info(k)
        assert (si["c"], si["p"], si["payload_bytes_per_warp"]) == (c, an.plans[c].p, an.plans[c].payload_bytes)
        assert si["live_bytes_per_warp"] == an.live[c].payload_bytes


@pytest.mark.parametrize("seed", range(60))
def test_analyzer_parity_random(seed):
    txt, _ = random_program(seed, loop=seed % 3 == 0, n_body=10)
    _same_plans(txt)


@pytest.mark.parametrize("seed", range(12))
def test_analyzer_parity_random_loop_nests(seed):
    txt, _ = random_program(700 + seed, loop=True, nested=True, n_body=8, indexed=seed % 3)
    _same_plans(txt)


def test_resume_code_of_a_loop_nest():
    """a site inside the inner loop of a nest resumes through
    RT_k and a peeled copy of the whole nest, whose branches to the nest's
    header go back to the normal code."""
    txt, _ = random_program(5, loop=True, nested=True, n_body=6)
    p = cb.Program(txt, debug=cb.DEBUG_FORCED | cb.DEBUG_NO_COMPILE)
    src = p.source
    assert "RT_" in src and "copy A of BB1..BB4" in src
    copy_a = src[src.index("copy A of BB1..BB4"):]
    copy_a = copy_a[:copy_a.index("\n}\n")]
    assert "goto BA2;" in copy_a and "goto BB1;" in copy_a and "goto BA1;" not in copy_a


@pytest.mark.parametrize("flags", [0, 1, 3, 5, 7])
def test_analyzer_parity_technique_toggles(flags):
    for seed in range(8):
        txt, _ = random_program(100 + seed, loop=seed % 2 == 0, n_body=9)
        _same_plans(txt, flags=flags)


@pytest.mark.parametrize("mode", [1, 2])
def test_analyzer_parity_live_full(mode):
    txt, _ = random_program(7, loop=True, n_body=9)
    _same_plans(txt, mode=mode)


def test_analyzer_parity_c1():
    _same_plans(configs.c1()["ir"])


def test_analyzer_parity_every_n():
    for seed in range(6):
        txt, _ = random_program(200 + seed, loop=True, n_body=14)
        _same_plans(txt, policy="EVERY_N")


def test_context_capacity_layout():
    p = cb.Program(configs.c1()["ir"], debug=cb.DEBUG_NO_COMPILE)
    info = p.info
    stride = ((info["max_payload_bytes_per_warp"] + 127) // 128) * 128
    for grid in (1, 7, 148):
        nw = grid * 4
        assert p.context_capacity(grid) == ((nw * 16 + 255) // 256) * 256 + nw * max(128, stride)


def test_runtime_options_generate_and_compile():
    """CTXB_GATHER_RESUME and CTXB_SYNC_POLL change only the generated code
    (plans identical); both compile for sm_100a with NVRTC."""
    from workloads import configs
    txt = configs.c4a_ir(1 << 14)
    base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT,
                      debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_AUTO_GATHER | cb.DEBUG_NO_AUTO_SIGNAL)
    g = cb.Program(txt, flags=cb.ALL | cb.GATHER_RESUME | cb.SYNC_POLL, poll_policy=cb.POLL_EXPLICIT)
    assert g.info["compiled"] == 1
    assert [g.plan_text(k) for k in range(g.num_sites)] == [base.plan_text(k) for k in range(base.num_sites)]
    src = g.source
    assert "resume_gather(P, lane, cta, dep" in src and "bar.sync 1" in src
    assert "__any_sync(0xffffffffu, sig_hit(ld_flag(flagp) == P.sig, fsrc, P, lane) != 0u)" in src
    assert "resume_gather(P" not in base.source and "sig_hit(ld_flag(flagp)" not in base.source
    assert "sig_hit(fl1, fsrc, P, lane)" in base.source


def test_host_signal_generates_and_compiles():
    """CTXB_HOST_SIGNAL changes only the generated poll sites
    (plans identical): relay warps load the host word with a system-scope load
    and forward it; it compiles for sm_100a alone and with CTXB_SYNC_POLL."""
    from workloads import configs
    txt = configs.c4a_ir(1 << 14)
    base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
    for extra in (0, cb.SYNC_POLL):
        h = cb.Program(txt, flags=cb.ALL | cb.HOST_SIGNAL | extra, poll_policy=cb.POLL_EXPLICIT)
        assert h.info["compiled"] == 1
        assert [h.plan_text(k) for k in range(h.num_sites)] == [base.plan_text(k) for k in range(base.num_sites)]
        src = h.source
        assert "ld.relaxed.sys.global.u32" in src and "relay_fwd(hfl, P, lane) != 0u)" in src
        assert "hfl = ld_hflag(hflagp); } else hfl = 0u;" in src
    assert "relay_fwd(hfl" not in base.source
    # forced (debug) programs ignore the option: no relay code is emitted
    f = cb.Program(txt, flags=cb.ALL | cb.HOST_SIGNAL, poll_policy=cb.POLL_EXPLICIT,
                   debug=cb.DEBUG_FORCED | cb.DEBUG_NO_COMPILE)
    assert "relay_fwd(hfl" not in f.source


def test_armed_signal_is_runtime_only():
    """CTXB_ARMED_SIGNAL is a runtime option: the generated
    kernel source is byte-identical to the default build's."""
    from workloads import configs
    txt = configs.c3()["ir"]
    dbg = cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_AUTO_SIGNAL   # the memop build, not the default watcher path
    base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=dbg)
    armed = cb.Program(txt, flags=cb.ALL | cb.ARMED_SIGNAL, poll_policy=cb.POLL_EXPLICIT, debug=dbg)
    assert armed.source == base.source
    with pytest.raises(cb.CtxbError):
        cb.Program(txt, flags=1 << 20, debug=cb.DEBUG_NO_COMPILE)


@pytest.mark.parametrize("flags", [cb.ALL, cb.ALL | cb.EXACT, cb.ALL | cb.RANK_RESUME | cb.PRUNE])
def test_parallel_analysis_equals_serial(flags, monkeypatch):
    """The per-site searches run on host threads (CTXB_ANALYZE_THREADS); plans,
    OSRB backups and exact-search counters equal the serial analysis."""
    txts = [configs.c4a_ir(1 << 14), configs.c3(512, 128, 64)["ir"]] + \
        [random_program(900 + s, loop=True, n_body=16)[0] for s in range(3)]
    for txt in txts:
        out = []
        for nt in ("1", "7"):
            monkeypatch.setenv("CTXB_ANALYZE_THREADS", nt)
            p = cb.Program(txt, flags=flags, debug=cb.DEBUG_NO_COMPILE)
            i = p.info
            out.append(([p.plan_text(k) for k in range(p.num_sites)], p.backups,
                        [i[k] for k in ("exact_windows", "exact_truncated", "exact_improved", "exact_fallback")]))
        assert out[0] == out[1]


def test_osrb_smem_slots_generate_and_compile():
    """CTXB_OSRB_SMEM moves the OSRB backup of C4a into a per-warp shared
    slot: plans unchanged, no bk register left, compiles for sm_100a."""
    txt = configs.c4a_ir(1 << 14)
    base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
    s = cb.Program(txt, flags=cb.ALL | cb.OSRB_SMEM, poll_policy=cb.POLL_EXPLICIT)
    assert s.info["compiled"] == 1 and s.backups == base.backups and s.backups
    assert [s.plan_text(k) for k in range(s.num_sites)] == [base.plan_text(k) for k in range(base.num_sites)]
    m = s.backups[0]
    assert "if (lane == 0u) BKS[warp][0] = " in s.source and "__syncwarp(); goto SAVE_SH_" in s.source
    assert f"u32 bk{m} " not in s.source
    assert f"u32 bk{m} = 0u;" in base.source


def test_osrb_lane_slots_generate_and_compile():
    """CTXB_OSRB_LANES: backup j in lane j of one register, read by a shuffle
    that every lane executes (hoisted out of the lane-select of the scalar
    store); exclusive with CTXB_OSRB_SMEM."""
    txt = configs.c4a_ir(1 << 14)
    s = cb.Program(txt, flags=cb.ALL | cb.OSRB_LANES, poll_policy=cb.POLL_EXPLICIT)
    assert s.info["compiled"] == 1 and s.backups
    src = s.source
    assert "BKV0 = lane == 0u ? " in src
    for line in src.split("\n"):
        if "__shfl_sync(0xffffffffu, BKV" in line:
            assert "if (lane ==" not in line, line
    with pytest.raises(cb.CtxbError):
        cb.Program(txt, flags=cb.ALL | cb.OSRB_LANES | cb.OSRB_SMEM, debug=cb.DEBUG_NO_COMPILE)


def test_flag_replicas_and_load_every_generate():
    """CTXB_FLAG_REPLICAS (master pollers forward to 64 replicas) and
    load_every (flag loads at every K-th poll visit): plans unchanged, both
    compile for sm_100a; the options reach the generated polls."""
    txt = configs.c3(512, 128, 64)["ir"]
    base = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_AUTO_SIGNAL)
    p = cb.Program(txt, flags=cb.ALL | cb.FLAG_REPLICAS, poll_policy=cb.POLL_EXPLICIT, load_every=4)
    assert p.info["compiled"] == 1
    assert [p.plan_text(k) for k in range(p.num_sites)] == [base.plan_text(k) for k in range(base.num_sites)]
    src = p.source
    assert "const u32 fsrc = gw % P.master_period == 0u ? 1u : 0u;" in src
    assert "if (--lcd == 0u) { lcd = 4u; fl1 = ld_flag(poll_addr(flagm, flagp, mcd)) == P.sig; }" in src
    assert "const u32 fsrc = 0u;" in base.source and "lcd" not in base.source
    with pytest.raises(cb.CtxbError):
        cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, load_every=4096, debug=cb.DEBUG_NO_COMPILE)


@pytest.mark.parametrize("rows", [2, 4])
def test_c3_unrolled_rows_parity(rows):
    """C3 with several stencil rows per loop iteration (the bench's C3): the
    same two kinds of poll site, C++ plans = oracle plans, the site after the
    advance still reverts."""
    txt = configs.c3_ir(512, 128, 64, rows_per_iter=rows)
    op = ir.parse(txt)
    an = A.analyze(op, policy="EXPLICIT")
    p = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
    assert p.num_sites == 2
    for k, c in enumerate(an.sites):
        assert p.plan_text(k) == A.plan_text(op, an.plans[c])
    assert an.plans[an.sites[1]].n_revert_pre + an.plans[an.sites[1]].n_revert_res > 0


def test_gather_resume_default_for_atomics():
    """resume launches gather by default in kernels with
    atomics (C4a, C4b), not otherwise (C1, C2); CTXB_DEBUG_NO_AUTO_GATHER and
    an explicit CTXB_GATHER_RESUME override it."""
    from workloads import configs
    cases = [(configs.c1()["ir"], 0), (configs.c2(128, 128, 64)["ir"], 0),
             (configs.c4a(1 << 14)["ir"], 1), (configs.c4b_ir(), 1)]
    for txt, want in cases:
        pol = cb.POLL_EXPLICIT if "poll" in txt else cb.POLL_EVERY_INSTR
        assert cb.Program(txt, poll_policy=pol, debug=cb.DEBUG_NO_COMPILE).info["gather_resume"] == want
        assert cb.Program(txt, poll_policy=pol, debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_AUTO_GATHER
                          ).info["gather_resume"] == 0
        assert cb.Program(txt, poll_policy=pol, flags=cb.ALL | cb.GATHER_RESUME,
                          debug=cb.DEBUG_NO_COMPILE).info["gather_resume"] == 1


def test_watcher_option_validation():
    """CTXB_WATCHER and CTXB_ARMED_SIGNAL both use the library's signal stream:
    exclusive.  The watcher changes no plan; the generated kernels only count
    their blocks' exits (so the watcher can end with its launch), without the
    drain notice's host store."""
    from workloads import configs
    txt = configs.c2(128, 128, 64)["ir"]
    with pytest.raises(cb.CtxbError) as e:
        cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | cb.WATCHER | cb.ARMED_SIGNAL,
                   debug=cb.DEBUG_NO_COMPILE)
    assert e.value.code == -1
    dbg = cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_AUTO_SIGNAL
    a = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, flags=cb.ALL | cb.WATCHER, debug=dbg)
    b = cb.Program(txt, poll_policy=cb.POLL_EXPLICIT, debug=dbg)
    assert [a.plan_text(k) for k in range(a.num_sites)] == [b.plan_text(k) for k in range(b.num_sites)]
    assert "warp_exit(P, lane, &blk_out)" in a.source and "warp_exit(P, lane, &blk_out)" not in b.source
    assert "#define CTXB_NOTICE_HOST 0" in a.source


def test_reexec_load_bytes():
    """ctxb_site_info_t.reexec_load_bytes_per_warp: C2's window re-executes the
    next k-step's 8 A and 8 B fragment loads (16 x 128 B, by hand from the IR:
    the software-pipelined prefetch precedes the poll); Fig 2's main block
    re-executes only ALU instructions (0 B), its init block its loads."""
    import json
    from workloads import configs
    p = cb.Program(configs.c2(256, 256, 64)["ir"], poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
    assert p.site_info(0)["reexec_load_bytes_per_warp"] == 16 * 128
    g = json.load(open(os.path.join(ROOT, "tests", "golden", "fig2.json")))
    q = cb.Program(g["ir"], debug=cb.DEBUG_NO_COMPILE)
    s0 = 6                                     # main: after the init block's 5 loads and its branch
    assert all(q.site_info(k)["reexec_load_bytes_per_warp"] == 0 for k in range(q.num_sites)
               if q.site_info(k)["c"] >= s0)
    assert q.site_info(1)["reexec_load_bytes_per_warp"] == 128      # re-executes `ldg v0, inp0[%tid]`
