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


# configs[1]: "tiled SGEMM-style IR kernel (register-heavy accumulators),
# 148 SMs x max resident blocks, random preemption points".
def c2_ir(M=4096, N=4096, K=4096, unroll=4, polls="iter"):
    """C = A.B, f32 row-major.  A 256-thread TB computes a 128x128 tile: thread
    (ty, tx) = (2*warp + lane/16, lane%16) owns rows row0+16i and columns
    col0+16j (i, j < 8) -> 64 accumulators v0..v63.  No shared memory.  Per k
    step a thread loads 8 A values and 8 B values into one of two fragment
    buffers (v64..v79 / v80..v95) and does 64 FFMAs.  The k loop is unrolled
    x`unroll` into one BB and software-pipelined: the fragments of step u+1 are
    loaded before the FFMAs of step u (the last prefetch of the final iteration
    is guarded off).  `poll` markers: polls="iter" -> one per iteration, after
    the last FFMA (its window spans the whole unrolled iteration); "step" ->
    before every step's FFMAs; "half" -> before and in the middle of every
    step's FFMAs.  Persistent grid: tile = ctaid + i*nctaid (reversible
    scalar IADD)."""
    assert M % 128 == 0 and N % 128 == 0 and K % unroll == 0 and unroll % 2 == 0
    tiles_n = N // 128
    ntiles = (M // 128) * tiles_n
    L = [".kernel c2_sgemm", ".buffer ro A", ".buffer ro B", ".buffer wo C",
         ".vregs 104", ".sregs 7", ".block 256"]
    frag = [(64, 72), (80, 88)]          # (A base, B base) of the two fragment buffers
    vA, vB, vT, vC, vty, vtx = 96, 97, 98, 99, 100, 101
    e = L.append

    def loads(buf, u, guard=""):
        a, b = frag[buf]
        g = f"@{guard} " if guard else ""
        for i in range(8):
            e(f"  iadd v{vT}, v{vA}, {16 * i * K + u}")
            e(f"  {g}ldg v{a + i}, A[v{vT}]")
        for j in range(8):
            e(f"  iadd v{vT}, v{vB}, {u * N + 16 * j}")
            e(f"  {g}ldg v{b + j}, B[v{vT}]")

    e("init:")
    e("  mov s0, %ctaid")                      # tile index
    e(f"  and v{vtx}, %laneid, 15")           # tx
    e(f"  shr v{vty}, %laneid, 4")
    e("  shl s1, %warpid, 1")
    e(f"  iadd v{vty}, v{vty}, s1")           # ty = 2*warp + lane/16
    e("tile:")
    e(f"  setp.lt.u s2, s0, {ntiles}")
    e("  brz s2, done")
    e("setup:")
    shift = tiles_n.bit_length() - 1
    e(f"  shr s3, s0, {shift}")                # tile_m
    e(f"  and s4, s0, {tiles_n - 1}")          # tile_n
    e("  shl s3, s3, 7")
    e("  shl s4, s4, 7")
    e(f"  iadd v{vT}, v{vty}, s3")             # row0
    e(f"  imul v{vA}, v{vT}, {K}")             # A index of (row0, k=0)
    e(f"  imul v{vC}, v{vT}, {N}")
    e(f"  iadd v{vB}, v{vtx}, s4")             # B index of (k=0, col0)
    e(f"  iadd v{vC}, v{vC}, v{vB}")           # C index of (row0, col0)
    for q in range(64):
        e(f"  mov v{q}, 0")
    loads(0, 0)                                # prologue: fragments of k = 0
    e(f"  mov s5, {K // unroll}")
    e("kloop:")
    e("  setp.ne.u s6, s5, 1")                 # a next iteration exists
    for u in range(unroll):
        cur, nxt = u % 2, (u + 1) % 2
        if u + 1 < unroll:
            loads(nxt, u + 1)
        else:
            loads(nxt, unroll, guard="s6")     # step 0 of the next iteration
        a, b = frag[cur]
        for q in range(64):
            if polls in ("step", "half") and q == 0:
                e("  poll")
            if polls == "half" and q == 32:
                e("  poll")
            i, j = q // 8, q % 8
            e(f"  ffma v{q}, v{a + i}, v{b + j}, v{q}")
    if polls == "iter":
        e("  poll")
    e(f"  iadd v{vA}, v{vA}, {unroll}")
    e(f"  iadd v{vB}, v{vB}, {unroll * N}")
    e("  isub s5, s5, 1")
    e("  brnz s5, kloop")
    e("store:")
    for q in range(64):
        i, j = q // 8, q % 8
        e(f"  iadd v{vT}, v{vC}, {16 * i * N + 16 * j}")
        e(f"  stg C[v{vT}], v{q}")
    e("  iadd s0, s0, %nctaid")
    e("  bra tile")
    e("done:")
    e("  exit")
    return "\n".join(L) + "\n"


def c2(M=4096, N=4096, K=4096, grid=None, polls="iter"):
    rA = np.random.default_rng(11)
    rB = np.random.default_rng(12)
    bufs = {
        "A": f32_bits(rA.uniform(-1.0, 1.0, M * K).astype(np.float32)),
        "B": f32_bits(rB.uniform(-1.0, 1.0, K * N).astype(np.float32)),
        "C": np.zeros(M * N, dtype=np.uint32),
    }
    # min_blocks: both generated kernels get __launch_bounds__(256, 2) so the
    # persistent grid keeps 2 resident blocks per SM (64 K registers / SM).
    return dict(name="C2", ir=c2_ir(M, N, K, polls=polls), grid=grid, min_blocks=2, buffers=bufs, uniforms={}, policy="EXPLICIT",
                M=M, N=N, K=K)


def bulk_ir(nvals=64, block=256):
    """Bulk save/restore microbench (SURVEY §8(d) '>=70 % gate'): every thread
    builds `nvals` live vector values from its thread id, then polls once; in
    forced mode every warp is preempted there and its LIVE context
    (nvals x 128 B per warp) goes through the generated save stub; the resume
    kernel's restore stub reads it back and the warp XOR-reduces the values
    (a guarded store that never fires keeps them live)."""
    n = nvals
    L = [".kernel bulk_ctx", ".buffer wo out", f".vregs {n + 1}", ".sregs 0", f".block {block}"]
    e = L.append
    for i in range(n):
        e(f"  xor v{i}, %tid, {hex(((i + 1) * 0x9E3779B9) & 0xFFFFFFFF)}")
    e("  poll")
    e(f"  xor v{n}, v0, v1")
    for i in range(2, n):
        e(f"  xor v{n}, v{n}, v{i}")
    e(f"  setp.eq.u v{n}, v{n}, 0x5A5A5A5B")
    e(f"  @v{n} stg out[%tid], v0")
    e("  exit")
    return "\n".join(L) + "\n"
