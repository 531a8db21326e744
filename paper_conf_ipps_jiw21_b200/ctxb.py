"""ctypes binding of libctxb (include/ctxb.h) -- argument marshalling only.

Every function named ``ctxb_*`` here calls the C entry point of the same name
(the boundary, include/ctxb.h); ``Program`` and ``Run`` are thin handle
wrappers over them.  Device memory and streams come from the caller (torch
tensors / streams, or raw integers); nothing is computed here.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

__all__ = [
    "LIB_PATH", "CtxbError", "lib",
    "RELAXED", "REVERT", "OSRB", "ALL", "DEFER", "PRUNE", "RANK_RESUME", "EXACT", "GATHER_RESUME", "SYNC_POLL", "HOST_SIGNAL", "ARMED_SIGNAL", "OSRB_SMEM", "OSRB_LANES", "FLAG_REPLICAS", "DRAIN_NOTICE", "WATCHER", "MODE_CTXBACK", "MODE_LIVE", "MODE_FULL", "MODE_FULL_HW",
    "POLL_EVERY_INSTR", "POLL_EVERY_N", "POLL_EXPLICIT",
    "DEBUG_FORCED", "DEBUG_POISON", "DEBUG_NO_POLLS", "DEBUG_NO_COMPILE", "DEBUG_NO_SHARE", "DEBUG_FENCE_STAMPS", "DEBUG_NO_AUTO_GATHER", "DEBUG_NO_FP_SHARE", "DEBUG_NO_SPEC_RESTORE",
    "DEBUG_NO_AUTO_SIGNAL", "DENSE_POLL_INSTRS",
    "STATE_NONE", "STATE_PREEMPTED", "STATE_DONE", "NEVER", "E_TIMEOUT", "EXPORTED_SYMBOLS",
    "ctxb_analyze", "ctxb_launch", "ctxb_preempt", "ctxb_resume", "ctxb_wait", "ctxb_context_bytes",
    "ctxb_flag_propagation", "ctxb_restore_floor",
    "Program", "Run",
]

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libctxb.so")

RELAXED, REVERT, OSRB, ALL, DEFER, PRUNE, RANK_RESUME, EXACT, GATHER_RESUME, SYNC_POLL, HOST_SIGNAL = \
    1, 2, 4, 7, 8, 16, 32, 64, 128, 256, 512
ARMED_SIGNAL, OSRB_SMEM, OSRB_LANES, FLAG_REPLICAS, DRAIN_NOTICE = 1024, 2048, 4096, 8192, 16384
WATCHER = 32768
MODE_CTXBACK, MODE_LIVE, MODE_FULL, MODE_FULL_HW = 0, 1, 2, 3
POLL_EVERY_INSTR, POLL_EVERY_N, POLL_EXPLICIT = 0, 1, 2
DEBUG_FORCED, DEBUG_POISON, DEBUG_NO_POLLS, DEBUG_NO_COMPILE, DEBUG_NO_SHARE = 1, 2, 4, 8, 16
DEBUG_FENCE_STAMPS, DEBUG_NO_AUTO_GATHER, DEBUG_NO_FP_SHARE, DEBUG_NO_SPEC_RESTORE = 32, 128, 256, 512
DEBUG_NO_AUTO_SIGNAL = 1024   # keep the caller's signal-path / poll-test bits (no defaults)
DENSE_POLL_INSTRS = 32        # sites on a loop shorter than this get the pipelined test + replicas
STATE_NONE, STATE_PREEMPTED, STATE_DONE = 0, 1, 2
NEVER = 0xFFFFFFFF
E_TIMEOUT = -8   # ctxb_preempt gave up waiting (env CTXB_PREEMPT_TIMEOUT_US)

EXPORTED_SYMBOLS = [
    "ctxb_last_error", "ctxb_version", "ctxb_analyze", "ctxb_program_destroy", "ctxb_program_info",
    "ctxb_num_sites", "ctxb_site_info", "ctxb_backups", "ctxb_site_plan_text", "ctxb_generated_source",
    "ctxb_occupancy", "ctxb_context_capacity", "ctxb_launch", "ctxb_preempt", "ctxb_resume", "ctxb_wait",
    "ctxb_query", "ctxb_flag_propagation", "ctxb_launch_ms", "ctxb_resume_stats_get", "ctxb_context_bytes", "ctxb_read_headers", "ctxb_read_stamps",
    "ctxb_run_destroy", "ctxb_preempt_async", "ctxb_program_cubin", "ctxb_restore_floor",
    "ctxb_persistent_grid",
]


class CtxbError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"ctxb error {code}: {msg}")
        self.code = code


class _Opts(C.Structure):
    _fields_ = [("flags", C.c_uint32), ("mode", C.c_uint32), ("poll_policy", C.c_uint32),
                ("poll_every", C.c_uint32), ("debug", C.c_uint32), ("flag_depth", C.c_uint32),
                ("min_blocks_per_sm", C.c_uint32), ("defer_instr_bytes", C.c_uint32),
                ("resume_level_bytes", C.c_uint32), ("exact_budget", C.c_uint32), ("load_every", C.c_uint32)]


class _SiteInfo(C.Structure):
    _fields_ = [(n, C.c_uint32) for n in ("c", "p", "n_vec", "n_scalar", "n_revert_pre", "n_revert_res",
                                          "n_reexec", "payload_bytes_per_warp", "live_bytes_per_warp",
                                          "defer_site", "reexec_load_bytes_per_warp")]


class _ProgInfo(C.Structure):
    _fields_ = [(n, C.c_uint32) for n in ("n_instrs", "nv", "ns", "block", "n_buffers", "n_uniforms", "n_sites",
                                          "n_backups", "max_payload_bytes_per_warp", "full_ir_bytes_per_warp",
                                          "num_regs", "compiled", "num_regs_resume", "resume_maxnreg",
                                          "n_save_stubs", "cubin_bytes", "exact_windows", "exact_truncated",
                                          "exact_improved", "exact_fallback")] + \
               [("analyze_ms", C.c_double), ("codegen_ms", C.c_double), ("compile_ms", C.c_double)] + \
               [(n, C.c_uint32) for n in ("spill_stores", "spill_loads", "spill_stores_resume", "spill_loads_resume",
                                          "gather_resume", "n_fp_shared", "flags", "poll_loop_instrs")]


class _PreStats(C.Structure):
    _fields_ = [("latency_us", C.c_double), ("host_us", C.c_double), ("signal_to_drained_us", C.c_double),
                ("warps_preempted", C.c_uint32),
                ("warps_done", C.c_uint32), ("blocks_preempted", C.c_uint32), ("payload_bytes", C.c_uint64),
                ("header_bytes", C.c_uint64)]


class _ResStats(C.Structure):
    _fields_ = [("resume_us", C.c_double), ("warps_resumed", C.c_uint32)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libctxb.so not built ({LIB_PATH}); run __graft_entry__.build() -- "
                          "there is no CPU fallback")
    L = C.CDLL(LIB_PATH)
    P, U32, U64, SZ, I = C.c_void_p, C.c_uint32, C.c_uint64, C.c_size_t, C.c_int
    sig = {
        "ctxb_last_error": (C.c_char_p, []),
        "ctxb_version": (C.c_char_p, []),
        "ctxb_analyze": (I, [C.c_char_p, SZ, C.POINTER(_Opts), C.POINTER(P)]),
        "ctxb_program_destroy": (I, [P]),
        "ctxb_program_info": (I, [P, C.POINTER(_ProgInfo)]),
        "ctxb_num_sites": (I, [P, C.POINTER(U32)]),
        "ctxb_site_info": (I, [P, U32, C.POINTER(_SiteInfo)]),
        "ctxb_backups": (I, [P, C.POINTER(U32), U32, C.POINTER(U32)]),
        "ctxb_site_plan_text": (I, [P, U32, I, C.c_char_p, SZ, C.POINTER(SZ)]),
        "ctxb_generated_source": (I, [P, C.c_char_p, SZ, C.POINTER(SZ)]),
        "ctxb_context_capacity": (I, [P, U32, C.POINTER(U64)]),
        "ctxb_occupancy": (I, [P, C.POINTER(U32), C.POINTER(U32)]),
        "ctxb_launch": (I, [P, U32, C.POINTER(P), C.POINTER(U32), P, U64, P, C.POINTER(U32), C.POINTER(P)]),
        "ctxb_preempt": (I, [P, P, C.POINTER(_PreStats)]),
        "ctxb_resume": (I, [P, P, C.POINTER(U32)]),
        "ctxb_wait": (I, [P, C.POINTER(I)]),
        "ctxb_resume_stats_get": (I, [P, C.POINTER(_ResStats)]),
        "ctxb_launch_ms": (I, [P, C.POINTER(C.c_float)]),
        "ctxb_query": (I, [P, C.POINTER(I)]),
        "ctxb_flag_propagation": (I, [P, U32, C.POINTER(C.c_double), C.POINTER(C.c_double)]),
        "ctxb_context_bytes": (I, [P, C.POINTER(U64), C.POINTER(U64), C.POINTER(U32)]),
        "ctxb_read_headers": (I, [P, C.POINTER(U32), U64]),
        "ctxb_read_stamps": (I, [P, C.POINTER(U64), U64]),
        "ctxb_run_destroy": (I, [P]),
        "ctxb_preempt_async": (I, [P, P]),
        "ctxb_program_cubin": (I, [P, P, SZ, C.POINTER(SZ)]),
        "ctxb_restore_floor": (I, [P, U32, U32, U32, U32, C.POINTER(C.c_double)]),
        "ctxb_persistent_grid": (I, [P, C.POINTER(U32)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


lib = _load()


def _chk(rc):
    if rc != 0:
        raise CtxbError(rc, lib.ctxb_last_error().decode(errors="replace"))


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return int(x.data_ptr())


def _stream(s):
    if s is None:
        return None
    if isinstance(s, int):
        return s
    return int(s.cuda_stream)


def _u32arr(vals):
    if vals is None:
        return None
    a = np.ascontiguousarray(np.asarray(vals, dtype=np.uint32))
    return a, a.ctypes.data_as(C.POINTER(C.c_uint32))


# --- the C-ABI names ----------------------------------------------------------

def ctxb_analyze(ir_text: str, flags=ALL, mode=MODE_CTXBACK, poll_policy=POLL_EVERY_INSTR, poll_every=8,
                 debug=0, flag_depth=1, min_blocks_per_sm=0, defer_instr_bytes=8,
                 resume_level_bytes=512, exact_budget=0) -> "Program":
    return Program(ir_text, flags, mode, poll_policy, poll_every, debug, flag_depth, min_blocks_per_sm,
                   defer_instr_bytes, resume_level_bytes, exact_budget)


def ctxb_launch(prog, grid, buffers, uniforms, ctx, stream=None, forced=None) -> "Run":
    return prog.launch(grid, buffers, uniforms, ctx, stream, forced)


def ctxb_preempt(run, ctrl_stream):
    return run.preempt(ctrl_stream)


def ctxb_resume(run, stream=None, forced=None):
    return run.resume(stream, forced)


def ctxb_wait(run):
    return run.wait()


def ctxb_context_bytes(run):
    return run.context_bytes()


def ctxb_flag_propagation(ctrl_stream, trials=20):
    """(median, max) us from the flag write on ctrl_stream to a spinning warp
    seeing it (device clock)."""
    m, x = C.c_double(), C.c_double()
    _chk(lib.ctxb_flag_propagation(_stream(ctrl_stream), trials, C.byref(m), C.byref(x)))
    return m.value, x.value


def ctxb_restore_floor(stream, bytes_per_warp, grid, block=256, trials=9):
    """Cold-read floor (us) of restoring bytes_per_warp (rounded up to 128) per
    warp on a grid x block launch: device span of a plain read of the same
    layout, L2 evicted before each trial."""
    m = C.c_double()
    b = (int(bytes_per_warp) + 127) // 128 * 128
    _chk(lib.ctxb_restore_floor(_stream(stream), b, grid, block, trials, C.byref(m)))
    return m.value


class Program:
    """An analysed + compiled IR kernel (ctxb_analyze)."""

    def __init__(self, ir_text, flags=ALL, mode=MODE_CTXBACK, poll_policy=POLL_EVERY_INSTR, poll_every=8,
                 debug=0, flag_depth=1, min_blocks_per_sm=0, defer_instr_bytes=8, resume_level_bytes=512,
                 exact_budget=0, load_every=1):
        self._h = C.c_void_p()
        self._pid = os.getpid()
        o = _Opts(flags, mode, poll_policy, poll_every, debug, flag_depth, min_blocks_per_sm, defer_instr_bytes,
                  resume_level_bytes, exact_budget, load_every)
        b = ir_text.encode()
        _chk(lib.ctxb_analyze(b, len(b), C.byref(o), C.byref(self._h)))
        self.debug = debug

    def __del__(self):
        # a forked child (e.g. a multiprocessing worker) does not own the handle
        if getattr(self, "_h", None) and getattr(self, "_pid", None) == os.getpid():
            lib.ctxb_program_destroy(self._h)
            self._h = None

    @property
    def info(self):
        i = _ProgInfo()
        _chk(lib.ctxb_program_info(self._h, C.byref(i)))
        return {k: getattr(i, k) for k, _ in _ProgInfo._fields_}

    @property
    def num_sites(self):
        n = C.c_uint32()
        _chk(lib.ctxb_num_sites(self._h, C.byref(n)))
        return n.value

    def site_info(self, k):
        s = _SiteInfo()
        _chk(lib.ctxb_site_info(self._h, k, C.byref(s)))
        return {n: getattr(s, n) for n, _ in _SiteInfo._fields_}

    @property
    def backups(self):
        n = C.c_uint32()
        _chk(lib.ctxb_backups(self._h, None, 0, C.byref(n)))
        a = (C.c_uint32 * max(1, n.value))()
        _chk(lib.ctxb_backups(self._h, a, n.value, C.byref(n)))
        return [a[i] for i in range(n.value)]

    def _text(self, fn, *args):
        ln = C.c_size_t()
        rc = fn(self._h, *args, None, 0, C.byref(ln))
        if rc not in (0, -7):
            _chk(rc)
        buf = C.create_string_buffer(ln.value)
        _chk(fn(self._h, *args, buf, ln.value, C.byref(ln)))
        return buf.value.decode()

    def plan_text(self, k, live=False):
        return self._text(lib.ctxb_site_plan_text, k, 1 if live else 0)

    @property
    def source(self):
        return self._text(lib.ctxb_generated_source)

    def cubin(self) -> bytes:
        """The compiled sm_100a cubin (ctxb_program_cubin)."""
        ln = C.c_size_t()
        rc = lib.ctxb_program_cubin(self._h, None, 0, C.byref(ln))
        if rc not in (0, -7):
            _chk(rc)
        buf = C.create_string_buffer(ln.value)
        _chk(lib.ctxb_program_cubin(self._h, buf, ln.value, C.byref(ln)))
        return buf.raw[:ln.value]

    def occupancy(self):
        """(resident blocks per SM, number of SMs) -> persistent grid = product."""
        a, n = C.c_uint32(), C.c_uint32()
        _chk(lib.ctxb_occupancy(self._h, C.byref(a), C.byref(n)))
        return a.value, n.value

    def persistent_grid(self):
        """Blocks of a persistent grid (ctxb_persistent_grid): every block
        resident at once, room left for the CTXB_WATCHER warp."""
        g = C.c_uint32()
        _chk(lib.ctxb_persistent_grid(self._h, C.byref(g)))
        return g.value

    def context_capacity(self, grid):
        b = C.c_uint64()
        _chk(lib.ctxb_context_capacity(self._h, grid, C.byref(b)))
        return b.value

    def launch(self, grid, buffers, uniforms, ctx, stream=None, forced=None, ctx_bytes=None):
        bufs = (C.c_void_p * max(1, len(buffers)))(*[_ptr(b) for b in buffers])
        uni = _u32arr(uniforms if uniforms else [0])
        f = _u32arr(forced)
        if ctx_bytes is None:
            ctx_bytes = ctx.numel() * ctx.element_size() if hasattr(ctx, "numel") else 0
        h = C.c_void_p()
        _chk(lib.ctxb_launch(self._h, grid, bufs, uni[1], _ptr(ctx), ctx_bytes, _stream(stream),
                             f[1] if f else None, C.byref(h)))
        return Run(h, self, grid, (buffers, ctx))


class Run:
    """One launch and its preempt / resume history (ctxb_launch)."""

    def __init__(self, h, prog, grid, keep):
        self._h = h
        self._pid = os.getpid()
        self.prog = prog
        self.grid = grid
        self._keep = keep          # keep the caller's tensors alive

    def __del__(self):
        if getattr(self, "_h", None) and getattr(self, "_pid", None) == os.getpid():
            lib.ctxb_run_destroy(self._h)
            self._h = None

    @property
    def n_warps(self):
        return self.grid * self.prog.info["block"] // 32

    def preempt(self, ctrl_stream, stats=True):
        """Raise the signal and wait until the launch drained (ctxb_preempt).
        stats=False passes NULL stats (no stamp read-back on the preemption
        path) and returns None: `finished` tells whether warps were
        preempted, drain_stats() computes the device numbers later."""
        if not stats:
            _chk(lib.ctxb_preempt(self._h, _stream(ctrl_stream), None))
            return None
        s = _PreStats()
        _chk(lib.ctxb_preempt(self._h, _stream(ctrl_stream), C.byref(s)))
        return {k: getattr(s, k) for k, _ in _PreStats._fields_}

    def preempt_async(self, ctrl_stream):
        """Raise the signal and return at once (ctxb_preempt_async); wait() /
        running() / finished observe the drain."""
        _chk(lib.ctxb_preempt_async(self._h, _stream(ctrl_stream)))

    def drain_stats(self):
        """Device numbers of the last preempted launch, from the headers and
        %globaltimer stamps (as ctxb_preempt computes them): warps / blocks
        preempted, payload bytes, routines span max t_saved - min t_flag_seen."""
        h = self.headers()
        pre = h[:, 2] == STATE_PREEMPTED      # a PREEMPTED header always belongs to the latest launch
        out = {"warps_preempted": int(pre.sum()), "payload_bytes": int(h[pre, 1].astype(np.uint64).sum()),
               "blocks_preempted": int(pre.reshape(self.grid, -1).any(axis=1).sum()), "latency_us": 0.0}
        if out["warps_preempted"]:
            st = self.stamps()[pre].astype(np.int64)
            out["latency_us"] = float(st[:, 1].max() - st[:, 0].min()) / 1e3
        return out

    def resume(self, stream=None, forced=None):
        f = _u32arr(forced)
        _chk(lib.ctxb_resume(self._h, _stream(stream), f[1] if f else None))

    def wait(self):
        fin = C.c_int()
        _chk(lib.ctxb_wait(self._h, C.byref(fin)))
        return bool(fin.value)

    def running(self):
        """Non-blocking: True while the current launch executes (ctxb_query)."""
        r = C.c_int()
        _chk(lib.ctxb_query(self._h, C.byref(r)))
        return bool(r.value)

    @property
    def finished(self):
        """After the current launch completed: every warp done (no preempted warp left)."""
        fin = C.c_int()
        _chk(lib.ctxb_wait(self._h, C.byref(fin)))
        return bool(fin.value)

    def launch_ms(self):
        """Device duration of the last launch (library-recorded CUDA events)."""
        f = C.c_float()
        _chk(lib.ctxb_launch_ms(self._h, C.byref(f)))
        return f.value

    def resume_stats(self):
        s = _ResStats()
        _chk(lib.ctxb_resume_stats_get(self._h, C.byref(s)))
        return {k: getattr(s, k) for k, _ in _ResStats._fields_}

    def context_bytes(self):
        p, h, n = C.c_uint64(), C.c_uint64(), C.c_uint32()
        _chk(lib.ctxb_context_bytes(self._h, C.byref(p), C.byref(h), C.byref(n)))
        return p.value, h.value, n.value

    def headers(self):
        a = np.zeros(self.n_warps * 4, dtype=np.uint32)
        _chk(lib.ctxb_read_headers(self._h, a.ctypes.data_as(C.POINTER(C.c_uint32)), a.size))
        return a.reshape(-1, 4)

    def stamps(self):
        a = np.zeros(self.n_warps * 4, dtype=np.uint64)
        _chk(lib.ctxb_read_stamps(self._h, a.ctypes.data_as(C.POINTER(C.c_uint64)), a.size))
        return a.reshape(-1, 4)

    def watcher_stamp(self):
        """%globaltimer at which the CTXB_WATCHER warp last raised the flag (0: never)."""
        a = np.zeros(self.n_warps * 4 + 1, dtype=np.uint64)
        _chk(lib.ctxb_read_stamps(self._h, a.ctypes.data_as(C.POINTER(C.c_uint64)), a.size))
        return int(a[-1])
