"""Exact IEEE-754 binary32 arithmetic on uint32 bit patterns (numpy, vectorised).

Test infrastructure only.  The IR's f32 ops are round-to-nearest-even with no
flush-to-zero and no contraction (the paper fixes no
precision, BASELINE.md "Precision").  numpy float32 +,-,* are IEEE RN with
subnormals, so they are used directly.  A fused multiply-add must round
once; computing a*b+c in float64 and rounding to float32 is a *double*
rounding and can be wrong, so ``ffma`` uses:

  1. a*b is exact in float64 (24+24 <= 53 significand bits);
  2. TwoSum(a*b, c) gives s = fl64(ab+c) and the exact error e;
  3. round-to-odd: if e != 0 and s has an even last bit, step s one ulp
     towards e (the exact value lies strictly between s and that neighbour);
  4. RN to float32.  Round-to-odd at 53 >= 24+2 bits followed by RN to 24
     bits equals a single RN rounding (Boldo & Melquiond, "Emulation of FMA
     and correctly rounded sums: proved algorithms using rounding to odd").

Pinned by tests/test_oracle_arith.py against exact rational arithmetic
(fractions.Fraction) and glibc ``fmaf``.
"""
import numpy as np

U32 = np.uint32


def f(x):
    return np.asarray(x, dtype=np.uint32).view(np.float32)


def u(x):
    return np.asarray(x, dtype=np.float32).view(np.uint32)


def fadd(a, b):
    with np.errstate(all="ignore"):
        return u(f(a) + f(b))


def fsub(a, b):
    with np.errstate(all="ignore"):
        return u(f(a) - f(b))


def fmul(a, b):
    with np.errstate(all="ignore"):
        return u(f(a) * f(b))


def ffma(a, b, c):
    """Correctly rounded fma(a, b, c) in binary32 (single rounding)."""
    with np.errstate(all="ignore"):
        a64 = f(a).astype(np.float64)
        b64 = f(b).astype(np.float64)
        c64 = f(c).astype(np.float64)
        p = a64 * b64                      # exact
        s = p + c64
        bb = s - p
        e = (p - (s - bb)) + (c64 - bb)    # TwoSum error, exact
        si = np.atleast_1d(s).view(np.int64).copy()
        s1 = np.atleast_1d(s).copy()
        e1 = np.atleast_1d(e)
        fix = (e1 != 0) & ((si & 1) == 0) & np.isfinite(s1)
        if np.any(fix):
            # step one ulp towards e: magnitude grows iff e has the sign of s
            up = np.sign(e1[fix]) == np.sign(s1[fix])
            si[fix] = np.where(up, si[fix] + 1, si[fix] - 1)
        r = si.view(np.float64).astype(np.float32)
        r = r.reshape(np.shape(s))
        return u(r)


def i2f(a):
    """cvt.rn.f32.s32"""
    return u(np.asarray(a, dtype=np.uint32).view(np.int32).astype(np.float32))


def u2f(a):
    """cvt.rn.f32.u32"""
    return u(np.asarray(a, dtype=np.uint32).astype(np.float32))


def f2i(a):
    """cvt.rzi.s32.f32: truncate, saturate to int32, NaN -> 0."""
    x = f(a).astype(np.float64)
    with np.errstate(all="ignore"):
        t = np.trunc(x)
        t = np.where(np.isnan(t), 0.0, t)
        t = np.clip(t, -2147483648.0, 2147483647.0)
    return t.astype(np.int64).astype(np.int32).view(np.uint32)
