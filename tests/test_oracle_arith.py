"""Pins of the oracle interpreter's arithmetic against independent definitions.

* f32 ops against exact rational arithmetic (fractions.Fraction) rounded to
  nearest-even binary32 by a from-scratch rounding routine, and ffma against
  glibc fmaf (a correctly rounded C99 routine);
* integer ops against Python big-int arithmetic mod 2^32;
* every R-5 inverse against its forward op (closed form: op^-1(op(x)) = x).
"""
import ctypes
import ctypes.util
import math
import struct
from fractions import Fraction

import numpy as np
import pytest

from oracle import fp32, interp
from oracle.ir import Opd, Instr
from oracle.analysis import revert_spec

M = 0xFFFFFFFF


def bits_to_frac(b):
    f = struct.unpack("<f", struct.pack("<I", b))[0]
    return Fraction(f)


def round_f32(x: Fraction) -> int:
    """Round an exact rational to binary32, nearest-even, with subnormals."""
    if x == 0:
        return 0
    sign = 0x80000000 if x < 0 else 0
    a = abs(x)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    e = max(e, -126)                   # subnormal range shares the min exponent
    q = a / (Fraction(2) ** (e - 23))  # scaled significand
    n = q.numerator // q.denominator
    rem = q - n
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and n % 2 == 1):
        n += 1
    if n == (1 << 24):
        n >>= 1
        e += 1
    if e > 127:
        return sign | 0x7F800000
    if n < (1 << 23):                   # subnormal
        return sign | n
    return sign | ((e + 127) << 23) | (n - (1 << 23))


def rand_finite(rng, n, emin=-30, emax=30):
    m = rng.integers(0, 1 << 23, n)
    e = rng.integers(emin + 127, emax + 127, n)
    s = rng.integers(0, 2, n)
    return ((s << 31) | (e << 23) | m).astype(np.uint32)


@pytest.mark.parametrize("op", ["fadd", "fsub", "fmul"])
def test_f32_binary_ops_exact(op):
    rng = np.random.default_rng(1)
    a = rand_finite(rng, 400)
    b = rand_finite(rng, 400)
    got = getattr(fp32, op)(a, b)
    for x, y, g in zip(a, b, got):
        fx, fy = bits_to_frac(int(x)), bits_to_frac(int(y))
        ex = {"fadd": fx + fy, "fsub": fx - fy, "fmul": fx * fy}[op]
        want = round_f32(ex)
        if ex == 0:
            assert int(g) & 0x7FFFFFFF == 0
        else:
            assert int(g) == want, (hex(x), hex(y))


def test_ffma_exact_vs_fraction_including_hard_cases():
    rng = np.random.default_rng(2)
    a = rand_finite(rng, 2000, -20, 20)
    b = rand_finite(rng, 2000, -20, 20)
    c = rand_finite(rng, 2000, -40, 40)
    # hard cases: c = -round(a*b) so the result is the tiny rounding residue;
    # and c chosen so a*b+c sits next to a rounding tie of binary32
    ab = fp32.fmul(a[:500], b[:500])
    c[:500] = ab ^ np.uint32(0x80000000)
    got = fp32.ffma(a, b, c)
    for x, y, z, g in zip(a, b, c, got):
        ex = bits_to_frac(int(x)) * bits_to_frac(int(y)) + bits_to_frac(int(z))
        if ex == 0:
            assert int(g) & 0x7FFFFFFF == 0
        else:
            assert int(g) == round_f32(ex), (hex(x), hex(y), hex(z))


def test_ffma_double_rounding_trap():
    """A case where fl32(fl64(a*b+c)) is wrong: a*b + c = 1 + 2^-24 + 2^-70 lies
    just above a binary32 tie; float64 rounds it onto the tie (1 + 2^-24) and
    the second rounding then goes to even (1.0), while the correct single
    rounding is 1 + 2^-23."""
    a = np.uint32(0x3F800001)      # 1 + 2^-23
    b = np.uint32(0x3F7FFFFF)      # 1 - 2^-24       -> a*b = 1 + 2^-24 - 2^-47
    c = np.uint32(0x28000001)      # 2^-47 (1 + 2^-23)
    ex = bits_to_frac(int(a)) * bits_to_frac(int(b)) + bits_to_frac(int(c))
    want = round_f32(ex)
    assert want == 0x3F800001
    naive = np.float32(np.float64(a.view(np.float32)) * np.float64(b.view(np.float32))
                       + np.float64(c.view(np.float32))).view(np.uint32)
    assert int(naive) != want          # the trap is real
    assert int(fp32.ffma(a, b, c)) == want


def test_ffma_vs_glibc_fmaf():
    libm = ctypes.CDLL(ctypes.util.find_library("m"))
    libm.fmaf.restype = ctypes.c_float
    libm.fmaf.argtypes = [ctypes.c_float] * 3
    rng = np.random.default_rng(3)
    a = rand_finite(rng, 3000, -60, 60)
    b = rand_finite(rng, 3000, -60, 60)
    c = rand_finite(rng, 3000, -120, 120)
    got = fp32.ffma(a, b, c)
    fa, fb, fc = a.view(np.float32), b.view(np.float32), c.view(np.float32)
    for i in range(len(a)):
        r = libm.fmaf(float(fa[i]), float(fb[i]), float(fc[i]))
        want = struct.unpack("<I", struct.pack("<f", r))[0]
        assert int(got[i]) == want


def test_conversions():
    rng = np.random.default_rng(4)
    x = rng.integers(0, 1 << 32, 2000, dtype=np.uint64).astype(np.uint32)
    for v, g in zip(x, fp32.i2f(x)):
        sv = int(v) - (1 << 32) if int(v) >= (1 << 31) else int(v)
        assert int(g) == round_f32(Fraction(sv))
    for v, g in zip(x, fp32.u2f(x)):
        assert int(g) == round_f32(Fraction(int(v)))
    fl = rand_finite(rng, 2000, -5, 40)
    for v, g in zip(fl, fp32.f2i(fl)):
        f = struct.unpack("<f", struct.pack("<I", int(v)))[0]
        t = max(-(1 << 31), min((1 << 31) - 1, math.trunc(f)))
        assert int(g) == (t & M)
    nan = np.uint32(0x7FC00000)
    assert int(fp32.f2i(nan)) == 0


INT_DEFS = {
    "iadd": lambda a, b: (a + b) & M,
    "isub": lambda a, b: (a - b) & M,
    "imul": lambda a, b: (a * b) & M,
    "and": lambda a, b: a & b,
    "or": lambda a, b: a | b,
    "xor": lambda a, b: a ^ b,
    "shl": lambda a, b: (a << b) & M if b < 32 else 0,
    "shr": lambda a, b: a >> b if b < 32 else 0,
    "sar": lambda a, b: ((a - (1 << 32) if a >> 31 else a) >> min(b, 31)) & M,
    "rotl": lambda a, b: ((a << (b % 32)) | (a >> (32 - b % 32))) & M if b % 32 else a,
    "rotr": lambda a, b: ((a >> (b % 32)) | (a << (32 - b % 32))) & M if b % 32 else a,
    "umin": min, "umax": max,
    "imin": lambda a, b: min(a - (a >> 31 << 32), b - (b >> 31 << 32)) & M,
    "imax": lambda a, b: max(a - (a >> 31 << 32), b - (b >> 31 << 32)) & M,
}


@pytest.mark.parametrize("op", sorted(INT_DEFS))
def test_integer_ops(op):
    rng = np.random.default_rng(hash(op) % 1000)
    a = rng.integers(0, 1 << 32, 500, dtype=np.uint64).astype(np.uint32)
    b = rng.integers(0, 1 << 32, 500, dtype=np.uint64).astype(np.uint32)
    b[:200] = rng.integers(0, 70, 200)
    got = interp.alu(op, (), [a, b])
    for x, y, g in zip(a, b, got):
        assert int(g) == INT_DEFS[op](int(x), int(y)), (op, x, y)


def test_imad_sel_setp_not_neg():
    rng = np.random.default_rng(9)
    a, b, c = (rng.integers(0, 1 << 32, 300, dtype=np.uint64).astype(np.uint32) for _ in range(3))
    for x, y, z, g in zip(a, b, c, interp.alu("imad", (), [a, b, c])):
        assert int(g) == (int(x) * int(y) + int(z)) & M
    for x, y, z, g in zip(a & 1, b, c, interp.alu("sel", (), [a & 1, b, c])):
        assert int(g) == (int(y) if x else int(z))
    for x, g in zip(a, interp.alu("not", (), [a])):
        assert int(g) == (~int(x)) & M
    for x, g in zip(a, interp.alu("neg", (), [a])):
        assert int(g) == (-int(x)) & M
    for cmp, fn in [("lt", lambda x, y: x < y), ("ge", lambda x, y: x >= y), ("eq", lambda x, y: x == y)]:
        for x, y, g in zip(a, b, interp.alu("setp", (cmp, "u"), [a, b])):
            assert int(g) == int(fn(int(x), int(y)))
        for x, y, g in zip(a, b, interp.alu("setp", (cmp, "s"), [a, b])):
            sx = int(x) - (1 << 32) if x >> 31 else int(x)
            sy = int(y) - (1 << 32) if y >> 31 else int(y)
            assert int(g) == int(fn(sx, sy))


REV_FORMS = [
    ("iadd", [("v", 0), ("v", 0), ("v", 1)]),
    ("iadd", [("v", 0), ("v", 1), ("v", 0)]),
    ("iadd", [("v", 0), ("v", 0), ("imm", 12345)]),
    ("isub", [("v", 0), ("v", 0), ("v", 1)]),
    ("isub", [("v", 0), ("v", 1), ("v", 0)]),
    ("xor", [("v", 0), ("v", 1), ("v", 0)]),
    ("imul", [("v", 0), ("v", 0), ("imm", 0x2545F491)]),
    ("imul", [("v", 0), ("imm", 7), ("v", 0)]),
    ("rotl", [("v", 0), ("v", 0), ("imm", 13)]),
    ("rotr", [("v", 0), ("v", 0), ("imm", 31)]),
    ("not", [("v", 0), ("v", 0)]),
    ("neg", [("v", 0), ("v", 0)]),
]


@pytest.mark.parametrize("op,form", REV_FORMS)
def test_inverses_roundtrip(op, form):
    """R-5: op^-1(op(r, R), R) == r for every reversible form, all inputs."""
    d = Opd(*form[0])
    srcs = [Opd(*f) for f in form[1:]]
    ins = Instr(op, d, srcs)
    spec = revert_spec(ins, "v0")
    assert spec is not None
    kind, others = spec
    rng = np.random.default_rng(11)
    r = rng.integers(0, 1 << 32, 1000, dtype=np.uint64).astype(np.uint32)
    x = rng.integers(0, 1 << 32, 1000, dtype=np.uint64).astype(np.uint32)
    vals = [r if s.reg == "v0" else (x if s.is_reg else np.uint32(s.val)) for s in srcs]
    rp = interp.alu(op, (), vals)
    oth = [x if o.is_reg else np.uint32(o.val) for o in others]
    assert np.array_equal(interp.invert(kind, rp, oth), r)


@pytest.mark.parametrize("op,form", [
    ("shl", [("v", 0), ("v", 0), ("imm", 3)]),          # bits lost
    ("imul", [("v", 0), ("v", 0), ("imm", 6)]),         # even multiplier
    ("imul", [("v", 0), ("v", 0), ("v", 1)]),           # unknown parity
    ("iadd", [("v", 0), ("v", 0), ("v", 0)]),           # r + r = 2r
    ("fadd", [("v", 0), ("v", 0), ("v", 1)]),           # rounding
    ("and", [("v", 0), ("v", 0), ("v", 1)]),
    ("shr", [("v", 0), ("v", 0), ("imm", 2)]),          # Fig 2 RSHL read as logical shift
])
def test_irreversible_forms(op, form):
    ins = Instr(op, Opd(*form[0]), [Opd(*f) for f in form[1:]])
    assert revert_spec(ins, "v0") is None
