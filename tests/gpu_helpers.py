"""Helpers for the GPU tests: run an IR kernel through the C-ABI (libctxb via
the ctypes binding) with forced per-warp preemption targets, and the oracle
on the same seeded inputs."""
from __future__ import annotations

import numpy as np

NEVER = 0xFFFFFFFF


def to_dev(arr):
    import torch
    a = np.ascontiguousarray(np.asarray(arr, dtype=np.uint32))
    return torch.from_numpy(a.view(np.int32).copy()).cuda()


def from_dev(t):
    return t.cpu().numpy().view(np.uint32).copy()


def gpu_run(prog, ir_prog_buffers_order, grid, buffers, uniforms, schedule=(), stream=None, max_launches=64):
    """Run `prog` (a paper_conf_ipps_jiw21_b200.Program compiled with
    DEBUG_FORCED) with schedule[k] = per-warp targets of launch k.  Returns
    (final buffers dict, list of per-launch header arrays)."""
    import torch
    names = ir_prog_buffers_order
    dev = {n: to_dev(buffers[n]) for n in names}
    cap = prog.context_capacity(grid)
    ctx = torch.zeros(cap, dtype=torch.uint8, device="cuda")
    nw = grid * prog.info["block"] // 32

    def targets(k):
        t = np.full(nw, NEVER, dtype=np.uint32)
        if k < len(schedule) and schedule[k] is not None:
            s = np.asarray(schedule[k], dtype=np.uint32)
            t[:len(s)] = s
        return t

    uni = [int(uniforms[u]) for u in uniforms] if uniforms else []
    run = prog.launch(grid, [dev[n] for n in names], uni, ctx, stream, forced=targets(0))
    headers = []
    k = 0
    while True:
        fin = run.wait()
        headers.append(run.headers().copy())
        if fin:
            break
        k += 1
        if k > max_launches:
            raise RuntimeError("too many launches")
        run.resume(stream, forced=targets(k))
    torch.cuda.synchronize()
    out = {n: from_dev(dev[n]) for n in names}
    return out, headers, run


def header_records(headers, epoch0=1):
    """Per launch: {warp: (site_k, live, bytes)} for warps preempted in it."""
    out = []
    for k, h in enumerate(headers):
        d = {}
        for w in range(h.shape[0]):
            if h[w, 2] == 1 and h[w, 3] == epoch0 + k:
                d[w] = (int(h[w, 0]) & 0x7FFFFFFF, bool(h[w, 0] >> 31), int(h[w, 1]))
        out.append(d)
    return out


def oracle_records(records, an):
    """Oracle preemption records -> per launch {warp: (site_k, live, bytes)}.
    A LIVE-fallback preemption (R-16) uses a separate stub only where the
    site's chosen plan is not already the LIVE plan (p < c)."""
    idx = {c: k for k, c in enumerate(an.sites)}
    out = {}
    for r in records:
        c = r["site"]
        live = r["kind"] == "live" and an.plans[c].p != c
        out.setdefault(r["launch"], {})[r["warp"]] = (idx[c], live, r["bytes"])
    n = max(out) + 1 if out else 0
    return [out.get(k, {}) for k in range(n)]


def flag_run(prog, grid, dev_buffers, uniforms, ctx, delay_s, stream, ctrl):
    """Launch, raise the preemption flag after `delay_s` (host clock), resume
    until done.  Returns the preempt stats (or None if the run finished
    first) and the header array of the preempted launch."""
    import time
    run = prog.launch(grid, dev_buffers, uniforms, ctx, stream)
    t0 = time.perf_counter()
    while time.perf_counter() < t0 + delay_s:
        pass
    st = run.preempt(ctrl)
    hdr = run.headers().copy()
    if st["warps_preempted"]:
        run.resume(stream)
        assert run.wait()
    return st, hdr, run


def check_headers_vs_plans(hdr, epoch, site_bytes, live_bytes):
    for w in range(hdr.shape[0]):
        if hdr[w, 2] == 1 and hdr[w, 3] == epoch:
            k, live = int(hdr[w, 0]) & 0x7FFFFFFF, bool(hdr[w, 0] >> 31)
            assert int(hdr[w, 1]) == (live_bytes[k] if live else site_bytes[k]), (w, hdr[w])
