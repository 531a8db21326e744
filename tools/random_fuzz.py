"""Extended GPU parity fuzz (beyond the test suite's 12 seeds): random IR
programs (workloads.randprog) in forced mode, poisoned resumes, every output
and every preempted warp's header checked against the oracle, over seeds and
analysis variants (CTXBack, LIVE, FULL_IR, FULL_HW, CTXB_PRUNE,
CTXB_RANK_RESUME, CTXB_EXACT, CTXB_DEFER).  Time-boxed.
Usage: python tools/random_fuzz.py first_seed n_seeds [seconds]"""
import os
import sys
import time
import traceback

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from oracle import ir  # noqa: E402
from test_gpu_baselines import check_mode  # noqa: E402
from test_gpu_parity import check  # noqa: E402
from workloads.randprog import random_buffers, random_program  # noqa: E402

VARIANTS = [("ctxback", 7, 0), ("live", 7, 1), ("full_ir", 7, 2), ("full_hw", 7, 3), ("prune", 7 | 16, 0),
            ("rank_resume", 7 | 32, 0), ("exact", 7 | 64, 0), ("ctxback_defer", 7 | 8, 0)]


def main(first, n, seconds):
    t_end = time.time() + seconds
    done, fails = 0, []
    for seed in range(first, first + n):
        if time.time() > t_end:
            break
        loop = seed % 3 == 0 or seed % 5 == 0
        nested = loop and seed % 2 == 0          # loop nests
        indexed = (seed // 2) % 3 if loop else 0  # loop-carried index bases (8r fast / generic path)
        txt, size = random_program(seed, loop=loop, nested=nested, indexed=indexed, n_body=10 + seed % 7)
        op = ir.parse(txt)
        grid = 1 + seed % 3
        nout = txt.count("stg out[")
        bufs = random_buffers(seed, op.block, grid, size, nout)
        r = np.random.default_rng(seed)
        nw = grid * op.nwarps
        scheds = [[r.integers(0, 90, nw).astype(np.uint32), r.integers(0, 30, nw).astype(np.uint32)]
                  for _ in range(3)]
        name, flags, mode = VARIANTS[seed % len(VARIANTS)]
        try:
            if mode:   # LIVE / FULL_IR / FULL_HW: the baselines' checker (FULL_HW bytes = 128 x NUM_REGS)
                check_mode(txt, grid, bufs, scheds, mode)
            else:
                check(txt, grid, bufs, scheds, flags=flags)
            done += 1
        except Exception:   # noqa: BLE001 -- report and continue
            fails.append((seed, name, traceback.format_exc(limit=3)))
            print(f"FAIL seed {seed} ({name})", flush=True)
    print(f"{done} programs passed, {len(fails)} failed (seeds {first}..{first + n - 1}, "
          f"variants cycled: {[v[0] for v in VARIANTS]})")
    for f in fails[:5]:
        print(f[0], f[1], f[2])
    return 1 if fails else 0


if __name__ == "__main__":
    a = sys.argv[1:]
    sys.exit(main(int(a[0]) if a else 1000, int(a[1]) if len(a) > 1 else 200, float(a[2]) if len(a) > 2 else 900))
