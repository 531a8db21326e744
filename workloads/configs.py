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
    the last FFMA (its window spans the whole unrolled iteration); "two" ->
    before the FFMAs of steps 0 and unroll/2 (two sites per iteration); "step" ->
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
            if (polls in ("step", "half") or (polls == "two" and u % (unroll // 2) == 0)) and q == 0:
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


# Resident blocks per SM for the bulk kernels: caps both generated kernels at
# the same register budget (77 / 76 registers, 24 warps per SM) so neither
# spills (the compiler's own choice rematerialises the values in the save
# kernel and spills 56 B in the resume kernel, profiles/r02_sass.md).
BULK_MIN_BLOCKS = 3


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


# configs[2]: "2D 5-point stencil IR kernel with loop-carried induction
# registers (exercises instruction reverting)".
def c3_ir(W=8192, H=8192, strip=64, polls="both", rows_per_iter=1):
    """y = 0.5*x + 0.125*(N + S + W + E) on interior points (f32, IR order:
    ((N + S) + W) + E, then * 0.125, then 0.5*x + that).  Thread per column,
    256 columns x `strip` rows per work item; persistent grid, item = ctaid +
    i*nctaid.  Per row: five loads around idx, the sum, then the loop-carried
    induction registers advance (idx += W, row += 1: reversible IADDs) and the
    finished value is written behind at idx - W.  Polls: in the middle of the
    sum, and after the advance (there CTXBack reverts idx += W at resume and
    re-executes the loads and the sum instead of saving the result).
    rows_per_iter = R > 1 unrolls R rows per loop iteration and keeps the two
    polls in its first row's sum and after its last row's advance (poll
    density / R: the same two kinds of site)."""
    assert W % 256 == 0 and H % strip == 0 and strip % rows_per_iter == 0
    ncb = W // 256
    items = ncb * (H // strip)
    L = [".kernel c3_stencil", ".buffer ro X", ".buffer wo Y", ".vregs 12", ".sregs 8", ".block 256"]
    e = L.append
    e("init:")
    e("  mov s6, %ctaid")                               # work item
    e("item:")
    e(f"  setp.lt.u s7, s6, {items}")
    e("  brz s7, done")
    e("setup:")
    e(f"  and s0, s6, {ncb - 1}")                       # column block
    shift = ncb.bit_length() - 1
    e(f"  shr s1, s6, {shift}")                         # strip index
    e("  shl s2, s0, 8")
    e("  iadd v0, s2, %tid")                            # col
    e(f"  imul s3, s1, {strip}")                        # row
    e("  setp.gt.u v1, v0, 0")
    e(f"  setp.lt.u v2, v0, {W - 1}")
    e("  and v1, v1, v2")                               # interior column
    e(f"  imad v3, s3, {W}, v0")                        # idx of (row, col)
    e(f"  mov s5, {strip // rows_per_iter}")
    e("rows:")
    for rr in range(rows_per_iter):
        first, last = rr == 0, rr == rows_per_iter - 1
        e("  setp.gt.u s4, s3, 0")                          # row > 0
        e(f"  setp.lt.u s2, s3, {H - 1}")                   # row < H-1
        e("  and s4, s4, s2")                               # interior row
        e("  and v11, v1, s4")                              # interior point
        e(f"  isub v4, v3, {W}")
        e("  @v11 ldg v5, X[v4]")                           # north
        e(f"  iadd v4, v3, {W}")
        e("  @v11 ldg v6, X[v4]")                           # south
        e("  isub v4, v3, 1")
        e("  @v11 ldg v7, X[v4]")                           # west
        e("  iadd v4, v3, 1")
        e("  @v11 ldg v8, X[v4]")                           # east
        e("  ldg v9, X[v3]")                                # centre
        e("  fadd v10, v5, v6")
        e("  fadd v10, v10, v7")
        if polls in ("both", "mid") and first:
            e("  poll")
        e("  fadd v10, v10, v8")
        e("  fmul v10, v10, 0f3E000000")                    # * 0.125
        e("  fmul v9, v9, 0f3F000000")                      # 0.5 * x
        e("  fadd v10, v9, v10")
        e(f"  iadd v3, v3, {W}")                            # idx += W   (reversible)
        e("  iadd s3, s3, 1")                               # row += 1   (reversible)
        if polls in ("both", "end") and last:
            e("  poll")
        e(f"  isub v4, v3, {W}")                            # write behind at the old idx
        e("  @v11 stg Y[v4], v10")
    e("  isub s5, s5, 1")
    e("  brnz s5, rows")
    e("next:")
    e("  iadd s6, s6, %nctaid")
    e("  bra item")
    e("done:")
    e("  exit")
    return "\n".join(L) + "\n"


# Poll placement the bench uses for C3 and C4b (profiles/r02_poll_placement.md):
# the cheapest placement measured that keeps each config's kind of site --
# C3: 8 stencil rows per loop iteration, one site after the last row's advance
# (the reverting site); C4b: the edge-chunk site (the OSRB site), polled
# through flag replicas.  Both keep the poll-site overhead <= 5 %.
BENCH_C3 = dict(rows_per_iter=8, polls="end")
BENCH_C4B_POLLS = "edge"


def c3(W=8192, H=8192, strip=64, polls="both", rows_per_iter=1):
    r = np.random.default_rng(21)
    bufs = {"X": f32_bits(r.uniform(0.0, 1.0, W * H).astype(np.float32)),
            "Y": np.zeros(W * H, dtype=np.uint32)}
    return dict(name="C3", ir=c3_ir(W, H, strip, polls, rows_per_iter), grid=None, buffers=bufs, uniforms={},
                policy="EXPLICIT", W=W, H=H, strip=strip, min_blocks=0)


def c3_numpy_reference(x_bits, W, H):
    """Textbook f32 5-point stencil in the IR's operation order (test pin)."""
    x = x_bits.view(np.float32).reshape(H, W)
    y = np.zeros((H, W), dtype=np.float32)
    n, s = x[:-2, 1:-1], x[2:, 1:-1]
    w, e = x[1:-1, :-2], x[1:-1, 2:]
    acc = ((n + s) + w) + e
    acc = acc * np.float32(0.125)
    y[1:-1, 1:-1] = x[1:-1, 1:-1] * np.float32(0.5) + acc
    return y.reshape(-1).view(np.uint32)


# configs[3]: "histogram + BFS-frontier IR kernels with scalar-operand-limited
# re-execution (exercises on-chip scalar backup)".
def c4a_ir(nkeys=1 << 28, per_lane=8, mid_polls=0):
    """256-bin histogram of u32 keys (bin = key >> 24) with global atomics
    into a per-block private copy of the bins (hist[ctaid*256 + bin]; the
    copies are summed afterwards) so that atomics on the same address only
    come from one block.  Warp-cooperative chunk loop: a warp handles chunks
    of 32*per_lane keys; the chunk base is a scalar loaded from `starts` (an
    irreversible uniform load that overwrites the base the chunk's key loads
    were addressed from -- the OSRB case).  One poll per chunk,
    after the next base is loaded and before the atomics."""
    chunk = 32 * per_lane
    assert nkeys % chunk == 0
    nch = nkeys // chunk
    L = [".kernel c4a_hist", ".buffer ro keys", ".buffer ro starts", ".buffer rw hist",
         f".vregs {1 + 2 * per_lane}", ".sregs 7", ".block 256"]
    e = L.append
    e("init:")
    e("  imad s0, %ctaid, %nwarps, %warpid")          # chunk index = global warp id
    e("  imul s1, %nctaid, %nwarps")                  # total warps
    e("  shl s6, %ctaid, 8")                          # this block's private bins
    e(f"  setp.lt.u s2, s0, {nch}")
    e("  brz s2, done")
    e("first:")
    e("  ldg s3, starts[s0]")                         # base of the first chunk
    e("loop:")
    e("  iadd v0, s3, %laneid")
    for j in range(per_lane):
        e(f"  ldg v{1 + j}, keys[v0]")
        if j + 1 < per_lane:
            e("  iadd v0, v0, 32")
    for j in range(per_lane):
        e(f"  shr v{1 + per_lane + j}, v{1 + j}, 24")
        e(f"  iadd v{1 + per_lane + j}, v{1 + per_lane + j}, s6")
    e("  iadd s0, s0, s1")                            # next chunk (reversible)
    e(f"  setp.lt.u s2, s0, {nch}")
    e(f"  umin s4, s0, {nch - 1}")
    e("  ldg s3, starts[s4]")                         # next base: irreversible scalar overwrite
    e("  poll")
    for j in range(per_lane):
        # mid_polls > 0: more sites inside the atomics (each after per_lane /
        # (mid_polls + 1) of them), for a shorter poll interval
        if mid_polls and j and j % (per_lane // (mid_polls + 1)) == 0:
            e("  poll")
        e(f"  atom.add _, hist[v{1 + per_lane + j}], 1")
    e("  brnz s2, loop")
    e("done:")
    e("  exit")
    return "\n".join(L) + "\n"


def c4a(nkeys=1 << 28, skewed=False, per_lane=8, grid=2, mid_polls=0):
    """`grid` = number of blocks the kernel is launched with (the hist buffer
    holds one 256-bin copy per block)."""
    chunk = 32 * per_lane
    if skewed:
        r = np.random.default_rng(32)
        u = r.random(nkeys, dtype=np.float64)
        keys = np.floor((u ** 4) * 4294967296.0).astype(np.uint64).clip(0, 0xFFFFFFFF).astype(np.uint32)
    else:
        r = np.random.default_rng(31)
        keys = r.integers(0, 1 << 32, nkeys, dtype=np.uint64).astype(np.uint32)
    starts = (np.arange(nkeys // chunk, dtype=np.uint64) * chunk).astype(np.uint32)
    bufs = {"keys": keys, "starts": starts, "hist": np.zeros(256 * grid, dtype=np.uint32)}
    return dict(name="C4a", ir=c4a_ir(nkeys, per_lane, mid_polls), grid=grid, buffers=bufs, uniforms={},
                policy="EXPLICIT", nkeys=nkeys, min_blocks=0)


def c4b_ir(polls="both"):
    """One level of a level-synchronous top-down BFS: warp per frontier vertex
    (scalar v, edge range [beg, end) from irreversible uniform loads), lanes
    over its edges; dist[u] claimed with atomicCAS(INF -> level+1) and newly
    discovered vertices pushed with atomicAdd on the next-frontier counter.
    Polls ("both"): after the vertex's loads and before each edge chunk's
    atomics; "vertex" / "edge" keep one of the two."""
    L = [".kernel c4b_bfs", ".buffer ro rowptr", ".buffer ro colidx", ".buffer ro front",
         ".buffer rw dist", ".buffer rw nextf", ".buffer rw nextcnt", ".uniform nf", ".uniform lvl1",
         ".vregs 6", ".sregs 8", ".block 256"]
    e = L.append
    e("init:")
    e("  imad s0, %ctaid, %nwarps, %warpid")          # frontier index = global warp id
    e("  imul s1, %nctaid, %nwarps")
    e("vloop:")
    e("  setp.lt.u s2, s0, %nf")
    e("  brz s2, done")
    e("vbody:")
    e("  ldg s3, front[s0]")                          # v          (irreversible)
    e("  ldg s4, rowptr[s3]")                         # beg        (irreversible)
    e("  iadd s5, s3, 1")
    e("  ldg s5, rowptr[s5]")                         # end        (irreversible, reads old s5)
    e("  mov s6, s4")                                 # e = beg
    if polls in ("both", "vertex"):
        e("  poll")
    e("eloop:")
    e("  setp.lt.u s7, s6, s5")
    e("  brz s7, vnext")
    e("ebody:")
    e("  iadd v0, s6, %laneid")
    e("  setp.lt.u v1, v0, s5")
    e("  @v1 ldg v2, colidx[v0]")                     # neighbour u
    if polls in ("both", "edge"):
        e("  poll")
    e("  @v1 atom.cas v3, dist[v2], 0xFFFFFFFF, %lvl1")
    e("  setp.eq.u v4, v3, 0xFFFFFFFF")
    e("  and v4, v4, v1")                             # newly discovered
    e("  @v4 atom.add v5, nextcnt[0], 1")
    e("  @v4 stg nextf[v5], v2")
    e("  iadd s6, s6, 32")
    e("  bra eloop")
    e("vnext:")
    e("  iadd s0, s0, s1")
    e("  bra vloop")
    e("done:")
    e("  exit")
    return "\n".join(L) + "\n"


def c4b_graph(n=1 << 22, avg_deg=16, seed=41):
    """Uniform random directed graph in CSR: out-degrees ~ Poisson(avg_deg)
    (i.e. ~avg_deg*n edges with uniformly random endpoints), destinations
    uniform.  Source vertex 0."""
    r = np.random.default_rng(seed)
    deg = r.poisson(avg_deg, n).astype(np.uint64)
    rowptr = np.zeros(n + 1, dtype=np.uint64)
    np.cumsum(deg, out=rowptr[1:])
    m = int(rowptr[-1])
    colidx = r.integers(0, n, m, dtype=np.uint64).astype(np.uint32)
    return rowptr.astype(np.uint32), colidx


def bfs_reference(rowptr, colidx, src=0):
    """Plain level-synchronous BFS (numpy) -> dist (0xFFFFFFFF unreached)."""
    n = len(rowptr) - 1
    dist = np.full(n, 0xFFFFFFFF, dtype=np.uint32)
    dist[src] = 0
    front = np.array([src], dtype=np.int64)
    lvl = 0
    rp = rowptr.astype(np.int64)
    while len(front):
        beg, end = rp[front], rp[front + 1]
        cnt = end - beg
        idx = np.repeat(beg - np.concatenate(([0], np.cumsum(cnt)[:-1])), cnt) + np.arange(cnt.sum())
        nb = colidx[idx].astype(np.int64)
        nb = np.unique(nb[dist[nb] == 0xFFFFFFFF])
        lvl += 1
        dist[nb] = lvl
        front = nb
    return dist


# configs[4]: "full-occupancy mixed suite on 1 B200 under a latency-sensitive
# arrival trace, plus 8 independent per-GPU instances".
def c5_arrivals(seconds, mean_ms=10.0, seed=51):
    """Poisson arrival times (s) of latency-sensitive jobs, mean gap mean_ms."""
    r = np.random.default_rng(seed)
    gaps = r.exponential(mean_ms / 1e3, int(seconds / (mean_ms / 1e3) * 3) + 16)
    t = np.cumsum(gaps)
    return t[t < seconds]


def c2s_ir(M=4096, N=4096, K=4096):
    """NEXT N2: C2 with shared-memory tiles and barriers.  Per k-tile of 8 the
    block stages A (128x8, stored k-major) and B (8x128) in shared memory
    (4 + 4 loads per thread), `bar`, every thread reads its 8 A and 8 B values
    per k from shared memory and does 64 FFMAs, `bar`.  Same k order and fma
    chain as C2, so C is bit-identical to C2's.  Preemption is block-uniform
    at the two barriers of each k-tile (their windows reach back to the
    previous barrier)."""
    assert M % 128 == 0 and N % 128 == 0 and K % 8 == 0
    tiles_n = N // 128
    ntiles = (M // 128) * tiles_n
    L = [".kernel c2s_sgemm_smem", ".buffer ro A", ".buffer ro B", ".buffer wo C",
         ".vregs 88", ".sregs 7", ".block 256", ".smem 2048"]
    a, b = 64, 72
    vA, vB, vT, vC, vty, vtx, vU, vS = 80, 81, 82, 83, 84, 85, 86, 87
    e = L.append
    e("init:")
    e("  mov s0, %ctaid")
    e(f"  and v{vtx}, %laneid, 15")
    e(f"  shr v{vty}, %laneid, 4")
    e("  shl s1, %warpid, 1")
    e(f"  iadd v{vty}, v{vty}, s1")                  # ty
    e("tile:")
    e(f"  setp.lt.u s2, s0, {ntiles}")
    e("  brz s2, done")
    e("setup:")
    shift = tiles_n.bit_length() - 1
    e(f"  shr s3, s0, {shift}")
    e(f"  and s4, s0, {tiles_n - 1}")
    e("  shl s3, s3, 7")                             # row0
    e("  shl s4, s4, 7")                             # col0
    # staging indices: A: row0 + tid%128, k0 + (tid/128)*4 + q ; B: k0 + tid/32, col0 + (tid%32)*4 + q
    e(f"  and v{vT}, %tid, 127")
    e(f"  iadd v{vA}, v{vT}, s3")
    e(f"  imul v{vA}, v{vA}, {K}")                   # A row base
    e(f"  shr v{vU}, %tid, 7")
    e(f"  shl v{vU}, v{vU}, 2")                      # (tid/128)*4
    e(f"  iadd v{vA}, v{vA}, v{vU}")                 # A index of (row, k0 + kq)
    e(f"  shl v{vS}, v{vU}, 7")                      # As offset: kq*128
    e(f"  iadd v{vS}, v{vS}, v{vT}")                 # As[kq][m]
    e(f"  shr v{vU}, %tid, 5")                       # kk = tid/32
    e(f"  imul v{vB}, v{vU}, {N}")
    e(f"  and v{vT}, %tid, 31")
    e(f"  shl v{vT}, v{vT}, 2")
    e(f"  iadd v{vB}, v{vB}, v{vT}")
    e(f"  iadd v{vB}, v{vB}, s4")                    # B index of (k0 + kk, col0 + 4*(tid%32))
    e(f"  shl v{vU}, v{vU}, 7")
    e(f"  iadd v{vU}, v{vU}, v{vT}")
    e(f"  iadd v{vU}, v{vU}, 1024")                  # Bs[kk][n] at 1024 + kk*128 + n
    e(f"  iadd v{vC}, v{vty}, s3")
    e(f"  imul v{vC}, v{vC}, {N}")
    e(f"  iadd v{vC}, v{vC}, v{vtx}")
    e(f"  iadd v{vC}, v{vC}, s4")                    # C index of (row0 + ty, col0 + tx)
    for q in range(64):
        e(f"  mov v{q}, 0")
    e(f"  mov s5, {K // 8}")
    e("ktile:")
    for q in range(4):                                # stage A: As[kq+q][m]
        e(f"  iadd v{vT}, v{vA}, {q}")
        e(f"  ldg v{a + q}, A[v{vT}]")
        e(f"  iadd v{vT}, v{vS}, {q * 128}")
        e(f"  sts v{vT}, v{a + q}")
    for q in range(4):                                # stage B: Bs[kk][n + q]
        e(f"  iadd v{vT}, v{vB}, {q}")
        e(f"  ldg v{b + q}, B[v{vT}]")
        e(f"  iadd v{vT}, v{vU}, {q}")
        e(f"  sts v{vT}, v{b + q}")
    e("  poll")
    e("  bar")
    for kk in range(8):
        for i in range(8):
            e(f"  iadd v{vT}, v{vty}, {kk * 128 + 16 * i}")
            e(f"  lds v{a + i}, v{vT}")
        for j in range(8):
            e(f"  iadd v{vT}, v{vtx}, {1024 + kk * 128 + 16 * j}")
            e(f"  lds v{b + j}, v{vT}")
        for q in range(64):
            i, j = q // 8, q % 8
            e(f"  ffma v{q}, v{a + i}, v{b + j}, v{q}")
    e(f"  iadd v{vA}, v{vA}, 8")
    e(f"  iadd v{vB}, v{vB}, {8 * N}")
    e("  isub s5, s5, 1")
    e("  poll")
    e("  bar")
    e("  brnz s5, ktile")
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


def c2s(M=4096, N=4096, K=4096):
    cfg = c2(M, N, K)
    cfg.update(name="C2s", ir=c2s_ir(M, N, K), min_blocks=2)
    return cfg
