"""The driver parses bench.py's one stdout line: it must stay under 2 KB and
carry the contract's keys (metric, value, unit, rooflines, cpu_baseline,
e2e with its copy bytes, clocks, gpu_launches, config.workload).  Checked on
the committed round-2 detail file (CPU only)."""
import json
import os

import bench

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "roofline", "roofline_restore", "cpu_baseline", "e2e",
        "gpu_launches", "clocks", "full_hw", "vs_full_hw_pct", "resume_us", "context_bytes_per_tb", "configs"]


def test_compact_line_fits_and_has_the_contract_keys():
    d = json.load(open(os.path.join(ROOT, "profiles", "r02_bench_detail.json")))
    line = bench.compact_line(d, "gpurun_out/bench_detail.json")
    text = json.dumps(line)
    assert len(text.encode()) <= 2000, len(text)
    for k in KEYS:
        assert k in line, k
    assert line["metric"] == json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
    for r in ("roofline", "roofline_restore"):
        assert set(line[r]) >= {"bound", "achieved", "peak", "unit", "frac", "traffic"}
    assert set(line["cpu_baseline"]) >= {"value", "unit", "cores", "kind", "sample"}
    assert set(line["e2e"]) >= {"value", "unit", "h2d_bytes_per_step", "d2h_bytes_per_step"}
    assert line["e2e"]["h2d_bytes_per_step"] > 0 and line["e2e"]["d2h_bytes_per_step"] > 0
    assert line["config"]["workload"] and line["higher_is_better"] is False
    assert set(line["clocks"]) >= {"sm_mhz", "sm_max_mhz", "reasons"}
