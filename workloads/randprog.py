"""Seeded random IR programs for property / parity tests (inputs only).

A program is: an `init` BB that loads every register from read-only buffers,
then 1-3 body blocks of random instructions (optionally one counted loop with
a scalar trip counter), then a `fin` BB that stores every register to a
write-only buffer and exits.  Memory indices are %tid, or a register masked to
the buffer size first, so accesses are always in bounds.  Float registers are
only produced from small integers (u2f of a 12-bit mask) and a tracked
magnitude bound keeps every f32 value finite (no NaN / Inf, R-14).
"""
from __future__ import annotations

import numpy as np

INT2 = ["iadd", "isub", "imul", "and", "or", "xor", "shl", "shr", "sar",
        "umin", "umax", "imin", "imax"]
REV = ["iadd", "isub", "xor", "imul_odd", "rotl", "not", "neg"]


class _Gen:
    def __init__(self, seed, nv, ns, n_body, loop, block, mem_ops, fp, atomics):
        self.r = np.random.default_rng(seed)
        self.nv, self.ns = nv, ns
        self.n_body = n_body
        self.loop = loop
        self.block = block
        self.mem_ops = mem_ops
        self.fp = fp
        self.atomics = atomics
        self.lines = []
        self.fmag = {}  # float-typed vector reg -> log2 magnitude bound

    def pick(self, seq):
        return seq[int(self.r.integers(len(seq)))]

    def vreg(self):
        return f"v{int(self.r.integers(self.nv))}"

    def sreg(self):
        return f"s{int(self.r.integers(self.ns))}" if self.ns else None

    def imm(self):
        k = int(self.r.integers(4))
        if k == 0:
            return str(int(self.r.integers(0, 32)))
        if k == 1:
            return hex(int(self.r.integers(0, 1 << 32)))
        return str(int(self.r.integers(1, 1000)))

    def src_v(self):
        k = int(self.r.integers(10))
        if k < 6:
            return self.vreg()
        if k < 8 and self.ns:
            return self.sreg()
        if k < 9:
            return self.imm()
        return self.pick(["%tid", "%laneid", "%ctaid", "%warpid"])

    def src_s(self):
        k = int(self.r.integers(10))
        if k < 7 and self.ns:
            return self.sreg()
        if k < 9:
            return self.imm()
        return self.pick(["%ctaid", "%warpid", "%nctaid"])

    def emit(self, s):
        self.lines.append("  " + s)

    def dst(self, d, op_float=None):
        if d.startswith("v"):
            if op_float is None:
                self.fmag.pop(d, None)
            else:
                self.fmag[d] = op_float

    def alu(self, scalar):
        d = self.sreg() if scalar else self.vreg()
        src = self.src_s if scalar else self.src_v
        k = int(self.r.integers(20))
        if k < 7:   # reversible-shaped r = op(r, x)
            op = self.pick(REV)
            if op == "imul_odd":
                self.emit(f"imul {d}, {d}, {int(self.r.integers(0, 1 << 31)) * 2 + 1}")
            elif op == "rotl":
                self.emit(f"rotl {d}, {d}, {int(self.r.integers(1, 32))}")
            elif op in ("not", "neg"):
                self.emit(f"{op} {d}, {d}")
            else:
                x = src()
                while x == d:
                    x = src()
                if op in ("iadd", "xor") and self.r.integers(2):
                    self.emit(f"{op} {d}, {x}, {d}")
                elif op == "isub" and self.r.integers(2):
                    self.emit(f"isub {d}, {x}, {d}")
                else:
                    self.emit(f"{op} {d}, {d}, {x}")
            self.dst(d)
        elif k < 15:
            op = self.pick(INT2)
            self.emit(f"{op} {d}, {src()}, {src()}")
            self.dst(d)
        elif k < 16:
            self.emit(f"mov {d}, {src()}")
            self.dst(d)
        elif k < 17:
            cmp = self.pick(["eq", "ne", "lt", "le", "gt", "ge"])
            self.emit(f"setp.{cmp}.{self.pick(['u', 's'])} {d}, {src()}, {src()}")
            self.dst(d)
        elif k < 18:
            self.emit(f"sel {d}, {src()}, {src()}, {src()}")
            self.dst(d)
        elif k < 19:
            self.emit(f"imad {d}, {src()}, {src()}, {src()}")
            self.dst(d)
        else:
            self.emit(f"{self.pick(['rotr', 'shl'])} {d}, {src()}, {int(self.r.integers(0, 40))}")
            self.dst(d)

    def fpop(self):
        d = self.vreg()
        fl = [r for r in self.fmag]
        k = int(self.r.integers(4))
        if k == 0 or len(fl) < 2:
            self.emit(f"and {d}, {self.vreg()}, 0xFFF")
            self.emit(f"u2f {d}, {d}")
            self.fmag[d] = 12
            return
        a, b = self.pick(fl), self.pick(fl)
        if k == 1 and self.fmag[a] + self.fmag[b] < 100:
            self.emit(f"fmul {d}, {a}, {b}")
            self.fmag[d] = self.fmag[a] + self.fmag[b] + 1
        elif k == 2:
            c = self.pick(fl)
            if self.fmag[a] + self.fmag[b] < 100 and self.fmag[c] < 100:
                self.emit(f"ffma {d}, {a}, {b}, {c}")
                self.fmag[d] = max(self.fmag[a] + self.fmag[b], self.fmag[c]) + 2
            else:
                self.emit(f"f2i {d}, {a}")
                self.fmag.pop(d, None)
        else:
            op = self.pick(["fadd", "fsub"])
            self.emit(f"{op} {d}, {a}, {b}")
            self.fmag[d] = max(self.fmag[a], self.fmag[b]) + 1

    def memop(self, nbuf_ro, size):
        k = int(self.r.integers(4 if self.atomics else 3))
        if k == 0 or k == 1:
            d = self.vreg() if (self.r.integers(3) or not self.ns) else self.sreg()
            buf = f"ro{int(self.r.integers(nbuf_ro))}" if k == 0 else "rw0"
            if d.startswith("s"):
                t = self.sreg()
                self.emit(f"and {t}, {self.src_s()}, {size - 1}")
                self.emit(f"ldg {d}, {buf}[{t}]")
            elif self.r.integers(2):
                self.emit(f"ldg {d}, {buf}[%tid]")
            else:
                t = self.vreg()
                self.emit(f"and {t}, {self.src_v()}, {size - 1}")
                self.fmag.pop(t, None)
                self.emit(f"ldg {d}, {buf}[{t}]")
            self.dst(d)
        elif k == 2:
            self.emit(f"stg scr[%tid], {self.src_v()}")
        else:
            d = self.vreg()
            self.emit(f"atom.add {d}, rw0[%laneid], {self.src_v()}")
            self.dst(d)


def random_program(seed: int, nv: int = 6, ns: int = 2, n_body: int = 12, loop: bool = False,
                   block: int = 64, mem_ops: bool = True, fp: bool = True, atomics: bool = False,
                   nblocks_hint: int = 2, nested: bool = False, indexed: int = 0):
    """Return IR text.  Buffers: ro0, ro1 (size = block*nblocks_hint), rw0
    (same size), scr (wo scratch), out (wo, (nv+ns) words per thread).
    loop: the first body block is a counted loop; nested (with loop): an
    outer counted loop (2 trips) around all body blocks, its header holding
    the inner loop's counter set-up (a loop nest, as in C2's tile / k loops).
    indexed (with loop): the loop body also loads through `iadd t, base, c`
    from loop-carried index registers advanced at the end of the body (C2's
    A / B index pattern); 1: a base in [0, size/2); 2: also a
    base with its top bit set whose `+ c` wraps (mod 2^32) into range."""
    g = _Gen(seed, nv, ns, n_body, loop, block, mem_ops, fp, atomics)
    size = 1
    while size < block * nblocks_hint:
        size *= 2
    ix = loop and indexed > 0
    vA, vW = f"v{nv + 1}", f"v{nv + 2}"
    half = max(1, size // 2)
    hdr = [".kernel rnd%d" % seed, ".buffer ro ro0", ".buffer ro ro1", ".buffer rw rw0",
           ".buffer wo scr", ".buffer wo out", f".vregs {nv}",
           f".sregs {ns + (1 if loop else 0) + (1 if loop and nested else 0)}",
           f".block {block}"]
    g.lines.append("init:")
    for i in range(nv):
        g.emit(f"ldg v{i}, ro{i % 2}[%tid]")
    for i in range(ns):
        g.emit(f"and s{i}, %ctaid, {size - 1}")
        g.emit(f"ldg s{i}, ro{i % 2}[s{i}]")
    if ix:
        g.emit(f"and {vA}, %tid, {half - 1}")
        if indexed > 1:
            g.emit(f"iadd {vW}, %laneid, 0xFFFFFFC0")
    ctr = f"s{ns}"
    nblk = 1 + int(g.r.integers(3))
    outer = f"s{ns + 1}" if (loop and nested) else None
    if outer:
        g.emit(f"mov {outer}, 2")
        g.lines.append("outer:")
    for b in range(nblk):
        is_loop = loop and b == 0
        if is_loop:
            g.emit(f"mov {ctr}, {2 + int(g.r.integers(3))}")
        g.lines.append(f"b{b}:")
        for _ in range(n_body):
            k = int(g.r.integers(10))
            if is_loop and ix and k < 3:
                t, d = g.vreg(), g.vreg()
                if indexed > 1 and k == 0:
                    g.emit(f"iadd {t}, {vW}, {64 + int(g.r.integers(0, 64))}")
                    g.emit(f"ldg {d}, ro1[{t}]")
                else:
                    g.emit(f"iadd {t}, {vA}, {int(g.r.integers(0, half))}")
                    g.emit(f"ldg {d}, ro0[{t}]")
                g.fmag.pop(t, None)
                g.dst(d)
                continue
            if mem_ops and k < 2:
                g.memop(2, size)
            elif fp and k < 4:
                g.fpop()
            else:
                g.alu(scalar=(ns > 0 and k == 9))
        if is_loop and ix:
            g.emit(f"iadd {vA}, {vA}, 1")
            g.emit(f"and {vA}, {vA}, {half - 1}")
        if is_loop:
            g.emit(f"isub {ctr}, {ctr}, 1")
            g.emit(f"brnz {ctr}, b{b}")
    if outer:
        g.emit(f"isub {outer}, {outer}, 1")
        g.emit(f"brnz {outer}, outer")
    g.lines.append("fin:")
    nout = nv + ns
    # store every register: out[tid * nout + k]; use a fresh index register
    # computed from %tid so no program register is disturbed before its store
    hdr[6] = f".vregs {nv + 1 + (2 if ix else 0)}"
    t = f"v{nv}"
    g.emit(f"imad {t}, %ctaid, %ntid, %tid")
    g.emit(f"imul {t}, {t}, {nout}")
    for i in range(nv):
        g.emit(f"stg out[{t}], v{i}")
        g.emit(f"iadd {t}, {t}, 1")
    for i in range(ns):
        g.emit(f"stg out[{t}], s{i}")
        g.emit(f"iadd {t}, {t}, 1")
    g.emit("exit")
    return "\n".join(hdr + g.lines) + "\n", size


def random_buffers(seed: int, block: int, grid: int, size: int, nout_per_thread: int):
    r = np.random.default_rng(seed)
    nthreads = block * grid
    return {
        "ro0": r.integers(0, 1 << 32, size, dtype=np.uint32),
        "ro1": r.integers(0, 1 << 32, size, dtype=np.uint32),
        "rw0": r.integers(0, 1 << 32, size, dtype=np.uint32),
        "scr": np.zeros(max(size, nthreads), dtype=np.uint32),
        "out": np.zeros(nthreads * nout_per_thread, dtype=np.uint32),
    }
