"""The kernels' division by a loop-invariant divisor (fop_device.cuh:div2_by)
gives the correctly rounded quotient, i.e. the same bits as IEEE division.

The device form is Markstein's correction: r = RN(1/d), q0 = RN(a r),
rem = RN(a - q0 d) (one FMA), q = RN(q0 + rem r) (one FMA); lanes outside the
theorem's range (d not in [2^-125, 2^125], |q0| not in [2^-100, FLT_MAX],
|a| < 2^-100: the remainder would be subnormal and inexact; a = 0 keeps q0)
fall back to __fdiv_rn.  This CPU test emulates each fp32 operation EXACTLY
(every intermediate below is exact in float64, each fp32 rounding is one
correctly rounded float64 -> float32 conversion or an explicit nearest-even
decision) and compares with RN32(a/d) = float32(float64(a)/float64(d)) (double
rounding is innocuous for division since 53 >= 2*24 + 2).

Exhaustive over every fp32 mantissa of a in [1, 2) for a set of divisors (the
quotient's behaviour is invariant under scaling a by a power of two while it
stays normal), plus random a, d over the whole in-range exponent span.
Not a test of the oracle: a pin of the product's fast form.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")

F32 = np.float32


def _rn_sum(q0, t):
    """RN32(q0 + t) for float32 q0 (as float64) and float64 t with |t| < 2 ulp(q0):
    nearest-even among q0 - 2ulp_dn .. q0 + 2ulp_up, decided by exact float64 compares."""
    q0f = q0.astype(F32)
    up1 = np.nextafter(q0f, F32(np.inf)).astype(np.float64)
    dn1 = np.nextafter(q0f, F32(-np.inf)).astype(np.float64)
    up2 = np.nextafter(up1.astype(F32), F32(np.inf)).astype(np.float64)
    dn2 = np.nextafter(dn1.astype(F32), F32(-np.inf)).astype(np.float64)
    cands = np.stack([dn2, dn1, q0, up1, up2])            # float32 values, exact in float64
    x = q0 + t                                           # may round in float64: compare exactly below
    # distance |c - (q0 + t)| = |(c - q0) - t|; c - q0 is exact (neighbours), the difference of two
    # float64 numbers of similar size with few bits is exact here (|t| and |c - q0| < 2^-20 |q0|)
    dist = np.abs((cands - q0) - t)
    best = np.argmin(dist, axis=0)
    dmin = dist[best, np.arange(dist.shape[1])]
    # ties: pick the candidate with an even mantissa
    tie = (dist == dmin).sum(axis=0) > 1
    res = cands[best, np.arange(dist.shape[1])]
    if tie.any():
        for i in np.nonzero(tie)[0]:
            for k in range(5):
                if dist[k, i] == dmin[i] and (np.array([cands[k, i]], F32).view(np.uint32)[0] & 1) == 0:
                    res[i] = cands[k, i]
    del x
    return res


def device_div(a, d):
    """Emulation of fop::div2_by on float32 arrays a (any) and scalar d in range."""
    a64 = a.astype(np.float64)
    d64 = np.float64(F32(d))
    if not (2.0 ** -125 <= abs(d64) <= 2.0 ** 125):     # div_by_ok(d) false: __fdiv_rn for the launch
        return ieee_div(a, d)
    r = np.float64(F32(1.0 / d64))                       # RN32(1/d): double rounding safe
    q0 = (a64 * r).astype(F32).astype(np.float64)         # a*r exact in float64 (48 bits)
    rem = (a64 - q0 * d64).astype(F32).astype(np.float64)  # q0*d exact; a - q0*d exact (cancellation)
    t = rem * r                                           # exact (48 bits)
    q = _rn_sum(q0, t)
    m = np.abs(q0)
    ok = (m >= 2.0 ** -100) & (m <= float(np.finfo(F32).max)) & (np.abs(a64) >= 2.0 ** -100)
    fb = (a64 / d64).astype(F32).astype(np.float64)       # __fdiv_rn
    return np.where(ok, q, np.where(a64 == 0, q0, fb)).astype(F32)


def ieee_div(a, d):
    return (a.astype(np.float64) / np.float64(F32(d))).astype(F32)


def _same(x, y):
    return np.array_equal(x.view(np.uint32), y.view(np.uint32))


def test_exhaustive_mantissas():
    a = (np.arange(1 << 23, dtype=np.uint32) | np.uint32(127 << 23)).view(F32)   # every float in [1, 2)
    for d in (3.0, 7.0, 10.0, 0.1, 768.0, 1.5e-5, 3.3e7, -1.0000001, 1.9999999, 1.0 / 3.0):
        got, ref = device_div(a, d), ieee_div(a, d)
        bad = np.nonzero(got.view(np.uint32) != ref.view(np.uint32))[0]
        assert bad.size == 0, (d, a[bad[:4]], got[bad[:4]], ref[bad[:4]])


def test_random_full_range():
    rng = np.random.default_rng(5)
    for _ in range(40):
        e = rng.integers(-124, 125)
        d = F32(rng.uniform(1, 2) * 2.0 ** e * rng.choice([-1, 1]))
        bits = rng.integers(0, 0xFF800000, size=200000, dtype=np.uint64).astype(np.uint32)
        a = bits.view(F32)
        a = a[np.isfinite(a)]
        got, ref = device_div(a, d), ieee_div(a, d)
        assert _same(got, ref), d


def test_special_values_take_the_exact_path():
    a = np.array([0.0, -0.0, 1.0, -1.0, np.inf, -np.inf, np.nan, 3e38, -3e38, 1e-40, 6e4], F32)
    for d in (2.0, 0.5, 1e-30, 3e-39):
        got, ref = device_div(a, d), ieee_div(a, d)
        assert np.array_equal(np.isnan(got), np.isnan(ref))
        m = ~np.isnan(ref)
        assert _same(got[m], ref[m]), d
