"""BASELINE.json configurations as IR kernels + seeded synthetic buffers.

Inputs only (see workloads/__init__.py).  Each function returns a dict with
the IR text, grid, buffers (numpy uint32, f32 data as bit patterns) and
uniform parameters.  Recipes: DESIGN.md "Inputs".
"""
from __future__ import annotations

import numpy as np

# configs[0]: "24-instruction straight-line IR kernel, 1 thread block x 128
# threads, preempted at every instruction".  One BB of 24 instructions mixing
# reversible integer ops (IADD / XOR / IMUL by an odd immediate), irreversible
# ones (SHL, FFMA), read-only and read-write loads, and an irreversible scalar
# overwrite (the OSRB case).
C1_IR = """\
.kernel c1_k24
.buffer ro in0
.buffer ro in1
.buffer rw rw0
.buffer wo out
.vregs 12
.sregs 4
.block 128
  mov v0, %tid
  ldg v1, in0[v0]
  ldg v2, in1[v0]
  mov s0, %ctaid
  iadd v3, v1, 0x9E3779B9
  xor v4, v3, v1
  imul v3, v3, 0x2545F491
  ldg v5, rw0[v0]
  shl v6, v5, 3
  ffma v7, v2, v2, 0f3F000000
  iadd v4, v4, v6
  ldg s1, in0[s0]
  iadd v8, v4, s1
  shl s1, s1, 2
  xor v8, v8, v3
  ffma v7, v7, v2, v2
  shl v11, v0, 3
  stg out[v11], v8
  iadd v11, v11, 1
  stg out[v11], v7
  iadd v11, v11, 1
  iadd v9, v6, s1
  stg out[v11], v9
  exit
"""


def f32_bits(x):
    return np.asarray(x, dtype=np.float32).view(np.uint32)


def c1():
    r1 = np.random.default_rng(1)
    r2 = np.random.default_rng(2)
    r3 = np.random.default_rng(3)
    bufs = {
        "in0": r1.integers(0, 1 << 32, 128, dtype=np.uint64).astype(np.uint32),
        "in1": f32_bits(r2.uniform(-1.0, 1.0, 128).astype(np.float32)),
        "rw0": r3.integers(0, 1 << 32, 128, dtype=np.uint64).astype(np.uint32),
        "out": np.zeros(128 * 8, dtype=np.uint32),
    }
    return dict(name="C1", ir=C1_IR, grid=1, buffers=bufs, uniforms={}, policy="EVERY_INSTR")


def c1_random_site_vectors(n=512, seed=7, nwarps=4, nsites=24):
    """512 random per-warp site vectors (seed 7): warp w is preempted at poll
    visit t[w] (= site t[w] in straight-line code)."""
    r = np.random.default_rng(seed)
    return r.integers(0, nsites, size=(n, nwarps)).astype(np.uint32)
