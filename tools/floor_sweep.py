"""Cold-read floor of a restore vs bytes per warp on C2's persistent grid
(296 x 256): intercept (launch ramp + first DRAM round trip) and slope
(bandwidth) of ctxb_restore_floor, to place the in-situ resume (DESIGN.md §6,
§11 "Cold-restore floor").  Usage: python tools/floor_sweep.py [grid]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_jiw21_b200 as cb  # noqa: E402

grid = int(sys.argv[1]) if len(sys.argv) > 1 else 296
s = torch.cuda.Stream()
xs, ys = [], []
print("| bytes / warp | total MB | floor µs | effective TB/s |")
print("|---|---|---|---|")
for b in (128, 512, 1024, 2048, 4096, 8704, 12288, 16384, 24576, 32768):
    t = cb.ctxb_restore_floor(s, b, grid, 256, 9)
    mb = b * grid * 8 / 1e6
    xs.append(mb)
    ys.append(t)
    print(f"| {b} | {mb:.1f} | {t:.2f} | {mb / t:.2f} |", flush=True)
k, c = np.polyfit(xs[3:], ys[3:], 1)
print(f"\nlinear fit over >= 2 KiB / warp: floor = {c:.2f} us + bytes / {1 / k:.2f} TB/s (marginal); "
      f"at 20.9 MB: {c + k * 20.9:.2f} us")
