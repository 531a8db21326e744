#!/usr/bin/env python
"""Benchmark of the CTXBack save / restore hot path on B200 (BASELINE.json).

Metric: "preemption latency us / resume us / context bytes per TB; save/restore
HBM GB/s".  Workload (configs[1]): the C2 tiled SGEMM IR kernel, 4096^3 f32,
on a persistent grid of 148 SMs x max resident blocks.  One step = launch C2,
raise the preemption signal at a random time U[0.05, 0.95] x T_uninterrupted,
drain every warp through its generated save stub (a2-a5), resume (a6-a8) and
run to completion; C is checked bit-exact against the uninterrupted run every
step.  `value` = median device preemption latency (max t_saved - min
t_flag_seen over preempted warps, %globaltimer).  The same steps are run
against the FULL_HW and LIVE baselines (same framework, same kernel).

Also reported: bulk save / restore bandwidth of the generated stubs (>= 1 GiB
of context, >> L2) against the measured HBM peak (roofline), poll overhead,
in-situ save GB/s, the oracle timed on host cores (cpu_baseline), and an
end-to-end run through the public API with pinned host buffers (e2e).

  python bench.py [--gpus N --steps K --warmup W] [--impl reference]
Under torchrun (N > 1) every rank runs an independent replica on its own GPU
(the path does not shard); rank 0
prints max-over-ranks times.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "preemption latency µs / resume µs / context bytes per TB; save/restore HBM GB/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ctxb", choices=["ctxb", "reference"])
    ap.add_argument("--size", type=int, default=4096)
    ap.add_argument("--bulk-mib", type=int, default=1024)
    ap.add_argument("--no-baselines", action="store_true")
    ap.add_argument("--no-oracle", action="store_true")
    ap.add_argument("--seed", type=int, default=100)
    return ap.parse_args()


# ---- distributed plumbing (replicas only) ------------------------------------

def dist_setup(args):
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return ws, rank, local


def barrier(ws):
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()


def allmax(ws, x):
    if ws <= 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# ---- clocks ------------------------------------------------------------------

class Clocks:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.gpu = gpu
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.seek(0)
        sm, mx, reasons = [], [], set()
        names = ["active", "hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.f.read().splitlines():
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx.append(float(parts[2]))
            except ValueError:
                continue
            for n, v in zip(names[1:], parts[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        os.unlink(self.f.name)
        load = [s for s in sm if s > 500] or sm
        return {"sm_mhz": float(np.median(load)) if load else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---- the GPU arm --------------------------------------------------------------

def make_c2(cb, size, mode, debug=0):
    """C2 with one poll site per k-loop iteration (its window spans the whole
    unrolled iteration) and 2 resident blocks / SM (__launch_bounds__)."""
    from workloads import configs
    ir_text = configs.c2_ir(size, size, size, polls="iter")
    return cb.Program(ir_text, poll_policy=cb.POLL_EXPLICIT, mode=mode, debug=debug, min_blocks_per_sm=2)


def spin_until(t):
    while time.perf_counter() < t:
        pass


def preempt_steps(cb, prog, grid, bufs, ctx, s, ctrl, ref, t_unint_s, fracs, ws, check=True):
    """Run len(fracs) preempt/resume steps; returns per-step records."""
    import torch
    dA, dB, dC = bufs
    recs = []
    for fr in fracs:
        barrier(ws)
        torch.cuda.synchronize()
        ev0 = torch.cuda.Event(enable_timing=True)
        ev1 = torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            ev0.record(s)
        t0 = time.perf_counter()
        run = prog.launch(grid, [dA, dB, dC], [], ctx, s)
        spin_until(t0 + fr * t_unint_s)
        st = run.preempt(ctrl)
        launches = 1
        rs = {"resume_us": 0.0, "warps_resumed": 0}
        run_ms = run.launch_ms()
        res_ms = None
        if st["warps_preempted"]:
            run.resume(s)
            run.wait()
            launches += 1
            rs = run.resume_stats()
            res_ms = run.launch_ms()
        with torch.cuda.stream(s):
            ev1.record(s)
        torch.cuda.synchronize()
        ok = bool(torch.equal(dC, ref)) if check else True
        recs.append(dict(frac=fr, latency_us=st["latency_us"], host_us=st["host_us"], resume_us=rs["resume_us"],
                         payload=st["payload_bytes"], header=st["header_bytes"], blocks=st["blocks_preempted"],
                         warps=st["warps_preempted"], done=st["warps_done"], step_ms=ev0.elapsed_time(ev1),
                         run_ms=run_ms, resume_ms=res_ms, launches=launches, ok=ok))
        if check and not ok:
            raise SystemExit("C differs from the uninterrupted run after preempt/resume")
        del run
    return recs


def summarize(recs):
    pre = [r for r in recs if r["warps"] > 0]
    lat = np.array([r["latency_us"] for r in pre]) if pre else np.array([0.0])
    res = np.array([r["resume_us"] for r in pre]) if pre else np.array([0.0])
    out = {
        "latency_us_median": float(np.median(lat)), "latency_us_p99": float(np.percentile(lat, 99)),
        "latency_us_max": float(lat.max()),
        "resume_us_median": float(np.median(res)), "resume_us_max": float(res.max()),
        "host_latency_us_median": float(np.median([r["host_us"] for r in pre])) if pre else 0.0,
        "preempted_steps": len(pre), "steps": len(recs),
    }
    if pre:
        bpt = [r["payload"] / max(1, r["blocks"]) for r in pre]
        out["context_bytes_per_tb"] = float(np.median(bpt))
        out["header_bytes_per_tb"] = float(np.median([r["header"] / max(1, r["blocks"]) for r in pre]))
        out["insitu_save_gbs_median"] = float(np.median([r["payload"] / (r["latency_us"] * 1e3)
                                                         for r in pre if r["latency_us"] > 0]))
    return out


def bulk_bandwidth(cb, mib, reps=5):
    """Bulk save / restore through the generated stubs: every warp of a grid
    much larger than the GPU saves 64 live vector values (8 KiB / warp) and the
    resume kernel restores them.  Durations from library-recorded CUDA events
    on the launching stream."""
    import torch
    from workloads import configs
    prog = cb.Program(configs.bulk_ir(64), poll_policy=cb.POLL_EXPLICIT, mode=cb.MODE_LIVE,
                      debug=cb.DEBUG_FORCED)
    per_warp = 64 * 128
    nw = (mib << 20) // per_warp
    grid = nw // 8
    nw = grid * 8
    out = torch.zeros(256, dtype=torch.int32, device="cuda")
    ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
    zeros = np.zeros(nw, np.uint32)
    never = np.full(nw, cb.NEVER, np.uint32)
    s = torch.cuda.Stream()
    save_ms, rest_ms = [], []
    for i in range(reps + 2):
        run = prog.launch(grid, [out], [], ctx, s, forced=zeros)
        assert not run.wait()
        a = run.launch_ms()
        pb, hb, _ = run.context_bytes()
        assert pb == nw * per_warp
        run.resume(s, forced=never)
        assert run.wait()
        b = run.launch_ms()
        if i >= 2:
            save_ms.append(a)
            rest_ms.append(b)
        del run
    payload = nw * per_warp
    hdr = nw * 16
    save_bytes = payload + hdr            # payload + PREEMPTED header
    rest_bytes = payload + 2 * hdr        # payload + header read + DONE header write
    return dict(grid=grid, warps=nw, payload_bytes=payload, save_ms=float(np.median(save_ms)),
                restore_ms=float(np.median(rest_ms)),
                save_gbs=save_bytes / (np.median(save_ms) * 1e6), restore_gbs=rest_bytes / (np.median(rest_ms) * 1e6),
                save_bytes=save_bytes, restore_bytes=rest_bytes)


def poll_overhead(cb, size, grid, bufs, reps=5):
    import torch
    out = {}
    for name, dbg in (("polls", 0), ("no_polls", cb.DEBUG_NO_POLLS)):
        prog = make_c2(cb, size, cb.MODE_CTXBACK, dbg)
        ctx = torch.empty(prog.context_capacity(grid), dtype=torch.uint8, device="cuda")
        ts = []
        for i in range(reps + 1):
            run = prog.launch(grid, list(bufs), [], ctx)
            run.wait()
            if i:
                ts.append(run.launch_ms())
            del run
        out[name] = float(np.median(ts))
    out["overhead_pct"] = 100.0 * (out["polls"] / out["no_polls"] - 1.0)
    return out


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic():
    """Per-launch DRAM traffic of the bulk save / restore kernels from the
    committed ncu --set full capture (profiles/), if present."""
    p = os.path.join(ROOT, "profiles", "ncu_bulk_traffic.json")   # written from round-1 ncu capture
    if os.path.exists(p):
        try:
            return json.load(open(p))
        except Exception:
            return {}
    return {}


def oracle_sample(steps=1, seed=0):
    """The oracle (plain Python SIMT interpreter + CTXB-R1 analysis) on a
    bounded sample of the same workload: C2 at M=N=K=256, thread block 0
    (8 warps, 1 of 4 tiles), all warps preempted at one poll visit, resumed
    to completion.  Latency analogue = host time spent in the oracle's
    preemption routine for the 8 warps (at-preempt reverts + context
    serialisation); resume analogue = time in its resume routine."""
    from oracle import analysis as A
    from oracle import interp, ir
    from workloads import configs
    cfg = configs.c2(256, 256, 256)
    op = ir.parse(cfg["ir"])
    t0 = time.perf_counter()
    an = A.analyze(op, policy="EXPLICIT")
    t_an = time.perf_counter() - t0
    rng = np.random.default_rng(seed)
    out = []
    ref = None
    for _ in range(steps):
        visit = int(rng.integers(8, 500))
        m = interp.Machine(an, 4, cfg["buffers"], blocks=[0])
        tp, tr = [], []
        orig_p, orig_r = m._preempt, m._resume

        def P(w, c, _o=orig_p):
            t = time.perf_counter()
            _o(w, c)
            tp.append(time.perf_counter() - t)

        def R(w, _o=orig_r):
            t = time.perf_counter()
            c = _o(w)
            tr.append(time.perf_counter() - t)
            return c
        m._preempt, m._resume = P, R
        t1 = time.perf_counter()
        mem = m.run([np.full(8, visit, np.uint32)])
        wall = time.perf_counter() - t1
        nbytes = sum(r["bytes"] for r in m.records)
        out.append(dict(visit=visit, latency_us=sum(tp) * 1e6, resume_us=sum(tr) * 1e6, bytes=nbytes,
                        wall_s=wall, warps=len(m.records)))
    return out, t_an


def gpu_arm(args):
    import torch
    import paper_conf_ipps_jiw21_b200 as cb
    from workloads import configs
    ws, rank, local = dist_setup(args)
    torch.cuda.set_device(local)
    size = args.size
    cfg = configs.c2(size, size, size)
    M = N = K = size
    progs = {"ctxback": make_c2(cb, size, cb.MODE_CTXBACK)}
    if not args.no_baselines:
        progs["live"] = make_c2(cb, size, cb.MODE_LIVE)
        progs["full_hw"] = make_c2(cb, size, cb.MODE_FULL_HW)
    bps, nsm = progs["ctxback"].occupancy()
    for p in progs.values():
        bps = min(bps, p.occupancy()[0])
    grid = bps * nsm
    dA = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
    dB = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
    dC = torch.zeros(M * N, dtype=torch.int32, device="cuda")
    s = torch.cuda.Stream()
    ctrl = torch.cuda.Stream()
    ctxs = {k: torch.empty(p.context_capacity(grid), dtype=torch.uint8, device="cuda") for k, p in progs.items()}
    # uninterrupted reference + its duration
    pr = progs["ctxback"]
    ts = []
    for i in range(3):
        run = pr.launch(grid, [dA, dB, dC], [], ctxs["ctxback"], s)
        assert run.wait()
        ts.append(run.launch_ms())
        del run
    t_unint_ms = float(np.median(ts))
    ref = dC.clone()
    rng = np.random.default_rng(args.seed + rank)
    fr_w = rng.uniform(0.05, 0.95, args.warmup)
    fr_t = rng.uniform(0.05, 0.95, args.steps)
    # ---- main timed loop: CTXBack ----
    preempt_steps(cb, pr, grid, (dA, dB, dC), ctxs["ctxback"], s, ctrl, ref, t_unint_ms / 1e3, fr_w, ws)
    clk = Clocks(local)
    clk.start()
    barrier(ws)
    torch.cuda.synchronize()
    recs = preempt_steps(cb, pr, grid, (dA, dB, dC), ctxs["ctxback"], s, ctrl, ref, t_unint_ms / 1e3, fr_t, ws)
    torch.cuda.synchronize()
    clocks = clk.stop()
    main = summarize(recs)
    # ---- baselines in the same framework (same fracs) ----
    base = {}
    for k in ("full_hw", "live"):
        if k in progs:
            preempt_steps(cb, progs[k], grid, (dA, dB, dC), ctxs[k], s, ctrl, ref, t_unint_ms / 1e3, fr_w[:1], ws)
            r = preempt_steps(cb, progs[k], grid, (dA, dB, dC), ctxs[k], s, ctrl, ref, t_unint_ms / 1e3, fr_t, ws)
            base[k] = summarize(r)
    # ---- static context sizes per TB ----
    nwb = 8
    sinfo = [pr.site_info(k) for k in range(pr.num_sites)]
    static = {
        "ctxback_bytes_per_tb_per_site": [nwb * x["payload_bytes_per_warp"] for x in sinfo],
        "live_bytes_per_tb_per_site": [nwb * x["live_bytes_per_warp"] for x in sinfo],
        "full_ir_bytes_per_tb": nwb * pr.info["full_ir_bytes_per_warp"],
        "full_hw_bytes_per_tb": nwb * 128 * progs.get("full_hw", pr).info["num_regs"],
        "num_regs": pr.info["num_regs"],
    }
    # ---- poll overhead, bulk roofline ----
    ovh = poll_overhead(cb, size, grid, (dA, dB, dC))
    bulk = bulk_bandwidth(cb, args.bulk_mib)
    peak, peak_src = peaks()
    traffic = ncu_traffic()
    # ---- e2e: public API with pinned host buffers, H2D/D2H inside the step ----
    hA = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).pin_memory()
    hB = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).pin_memory()
    hC = torch.empty(M * N, dtype=torch.int32).pin_memory()
    e2e = []
    for fr in fr_t[:max(3, min(args.steps, 8))]:
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with torch.cuda.stream(s):
            dA.copy_(hA, non_blocking=True)
            dB.copy_(hB, non_blocking=True)
        s.synchronize()            # the flag time is relative to the kernel, not the copies
        run = pr.launch(grid, [dA, dB, dC], [], ctxs["ctxback"], s)
        spin_until(time.perf_counter() + fr * t_unint_ms / 1e3)
        st = run.preempt(ctrl)
        if st["warps_preempted"]:
            run.resume(s)
            run.wait()
        with torch.cuda.stream(s):
            hC.copy_(dC, non_blocking=True)
        s.synchronize()
        e2e.append(dict(host_us=st["host_us"], step_s=time.perf_counter() - t0, pre=st["warps_preempted"]))
        del run
    assert torch.equal(hC, ref.cpu()), "e2e result differs"
    e2e_val = float(np.median([x["host_us"] for x in e2e if x["pre"]] or [0.0]))
    # ---- max over ranks ----
    value = allmax(ws, main["latency_us_median"])
    ms_per_step = allmax(ws, float(np.mean([r["step_ms"] for r in recs])))
    launches = int(sum(r["launches"] for r in recs))
    if rank != 0:
        return None
    cpu = None
    if not args.no_oracle:
        samp, t_an = oracle_sample(1, args.seed)
        cpu = {"value": samp[0]["latency_us"], "unit": "us", "cores": 1, "kind": "oracle",
               "resume_us": samp[0]["resume_us"], "context_bytes_per_tb": samp[0]["bytes"],
               "sample": (f"C2 IR at M=N=K=256, thread block 0 (8 warps) preempted at poll visit "
                          f"{samp[0]['visit']} and resumed to completion on 1 host core; value = host time "
                          f"in the oracle's preemption routine for the 8 warps (analysis {t_an:.1f} s, "
                          f"interpretation {samp[0]['wall_s']:.1f} s, not counted)")}
    rf = {"kernel": "ctxb_run of the bulk IR kernel (generated save stub, 64 live vector values/warp)",
          "bound": "hbm", "achieved": round(bulk["save_gbs"], 1), "peak": peak, "unit": "GB/s",
          "frac": round(bulk["save_gbs"] / peak, 4), "traffic": traffic.get("save_traffic_per_launch"),
          "algorithmic_bytes_per_launch": bulk["save_bytes"], "peak_source": peak_src}
    rr = {"kernel": "ctxb_resume of the bulk IR kernel (generated restore stub)", "bound": "hbm",
          "achieved": round(bulk["restore_gbs"], 1), "peak": peak, "unit": "GB/s",
          "frac": round(bulk["restore_gbs"] / peak, 4), "traffic": traffic.get("restore_traffic_per_launch"),
          "algorithmic_bytes_per_launch": bulk["restore_bytes"], "peak_source": peak_src}
    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "us", "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": False,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"C2 tiled SGEMM IR kernel {M}x{N}x{K} f32 (configs[1]), persistent grid "
                               f"{nsm} SMs x {bps} blocks x 256 threads, flag at U[0.05,0.95] x T_uninterrupted",
                   "grid": grid, "block": 256, "t_uninterrupted_ms": round(t_unint_ms, 3),
                   "l2": "inputs larger than L2 (A, B, C = 192 MiB > 126 MB)", "parallelism": f"replicas x{ws}"},
        "resume_us": round(main["resume_us_median"], 3),
        "context_bytes_per_tb": main.get("context_bytes_per_tb"),
        "ctxback": main, "baselines": base, "static_context": static,
        "reduction_vs_full_hw": {
            "latency_pct": (round(100 * (1 - main["latency_us_median"] / base["full_hw"]["latency_us_median"]), 2)
                            if "full_hw" in base and base["full_hw"]["latency_us_median"] else None),
            "resume_pct": (round(100 * (1 - main["resume_us_median"] / base["full_hw"]["resume_us_median"]), 2)
                           if "full_hw" in base and base["full_hw"]["resume_us_median"] else None),
            "context_pct": (round(100 * (1 - main["context_bytes_per_tb"] / base["full_hw"]["context_bytes_per_tb"]), 2)
                            if "full_hw" in base and base["full_hw"].get("context_bytes_per_tb") and
                            main.get("context_bytes_per_tb") else None)},
        "poll_overhead": ovh, "bulk": bulk,
        "roofline": rf, "roofline_restore": rr,
        "cpu_baseline": cpu,
        "e2e": {"value": round(e2e_val, 3), "unit": "us",
                "what": "host-clock preemption latency of ctxb_preempt with inputs copied from pinned host "
                        "memory and C copied back every step",
                "h2d_bytes_per_step": 2 * M * K * 4, "d2h_bytes_per_step": M * N * 4},
        "gpu_launches": launches, "clocks": clocks,
        "parity": "C bit-exact vs the uninterrupted run in every step",
    }
    return line


def reference_arm(args):
    """--impl reference: the oracle (this task's reference arm) on host cores,
    rank 0 only; other ranks exit without work."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return None
    samp, t_an = oracle_sample(args.warmup + args.steps, args.seed)
    timed = samp[args.warmup:]
    v = float(np.median([x["latency_us"] for x in timed]))
    wall = sum(x["wall_s"] for x in timed)
    return {"impl": "reference", "metric": METRIC, "value": round(v, 3), "unit": "us", "n_gpus": 0,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * wall / max(1, len(timed)), 3),
            "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": f"C2 tiled SGEMM IR kernel {args.size}^3 (configs[1]) -- bounded oracle sample",
                       "sample": "M=N=K=256, thread block 0 (8 warps), random poll visit per step"},
            "resume_us": round(float(np.median([x["resume_us"] for x in timed])), 3),
            "cpu_baseline": {"value": round(v, 3), "unit": "us", "cores": 1, "kind": "oracle",
                             "sample": "C2 IR at M=N=K=256, TB 0 (8 warps), preempted at a random poll visit "
                                       "per step; value = host time in the oracle's preemption routine"},
            "e2e": {"value": round(v, 3), "unit": "us", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def main():
    args = parse()
    line = reference_arm(args) if args.impl == "reference" else gpu_arm(args)
    if line is not None:
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
