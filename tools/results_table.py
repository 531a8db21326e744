"""The per-config results table of README.md / DESIGN.md §8, printed from a
bench detail file (`bench.py --detail`, default gpurun_out/bench_detail.json;
the committed one is profiles/r02_bench_detail.json).  CPU only.
Usage: python tools/results_table.py [detail.json]"""
import json
import sys


def pct(a, b):
    if not (a and b):
        return ""
    r = 100 * (a / b - 1)
    return f"{r:.1f} %" if r < -99 else f"{r:.0f} %"


def kb(x):
    return f"{x / 1000:.1f} KB" if x >= 1000 else f"{x:.0f} B"


def row(name, cb, fh, ovh):
    cells = [name]
    cells.append(f"{cb['latency_us_median']:.2f} / {fh['latency_us_median']:.2f} µs "
                 f"({pct(cb['latency_us_median'], fh['latency_us_median'])})")
    h1, h2 = cb.get("host_latency_us_median"), fh.get("host_latency_us_median")
    cells.append(f"{h1:.2f} / {h2:.2f} µs ({pct(h1, h2)})" if h1 and h2 else "—")
    cells.append(f"{cb['resume_us_median']:.2f} / {fh['resume_us_median']:.2f} µs "
                 f"({pct(cb['resume_us_median'], fh['resume_us_median'])})")
    c1, c2 = cb.get("context_bytes_per_tb"), fh.get("context_bytes_per_tb")
    cells.append(f"{kb(c1)} / {kb(c2)} ({pct(c1, c2)})" if c1 and c2 else "")
    cells.append(f"{ovh:.1f} %" if ovh is not None else "—")
    return "| " + " | ".join(cells) + " |"


def main():
    path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/bench_detail.json"
    d = json.load(open(path))
    print("| config | routines CTXBack / FULL_HW | host latency CTXBack / FULL_HW | resume CTXBack / FULL_HW "
          "| context / TB CTXBack / FULL_HW | poll overhead |")
    print("|---|---|---|---|---|---|")
    cf = d.get("configs", {})
    names = {"c1": "C1 (24 sites, forced)", "c2s": "C2s SGEMM + smem tiles",
             "c3": "C3 stencil 8192^2 (8 rows/iter, reverting site)", "c4a": "C4a histogram 2^28 (gathered)",
             "c4b": "C4b BFS 2^22 (edge sites, replicas, gathered)"}
    if "c1" in cf:
        print(row(names["c1"], cf["c1"]["ctxback"], cf["c1"]["full_hw"], None))
    print(row(f"C2 SGEMM 4096^3 ({d.get('signal', 'watcher')} path)", d["ctxback"], d["baselines"]["full_hw"],
              d["poll_overhead"]["overhead_pct"]))
    for k in ("armed", "memop"):
        b = d["baselines"]
        if "ctxback_" + k in b:
            print(f"| C2 ({k}) | | {b['ctxback_' + k]['host_latency_us_median']:.1f} / "
                  f"{b['full_hw_' + k]['host_latency_us_median']:.1f} µs | | | |")
    for c in ("c2s", "c3", "c4a", "c4b"):
        if c in cf:
            print(row(names[c], cf[c]["ctxback"], cf[c]["full_hw"], cf[c]["poll_overhead"]["overhead_pct"]))
    if "c5" in cf:
        m = cf["c5"]["modes"]
        print("\nC5 LS wait p50 (ms):", {k: v["ls_wait_ms_p50"]
                                          for k, v in m.items()})


if __name__ == "__main__":
    main()
