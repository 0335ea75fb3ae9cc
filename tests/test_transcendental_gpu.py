"""GPU parity of every transcendental opcode and of the fast forms, on special
values and wide sweeps (the CUDA path through the C ABI vs the oracle).

Tolerances, each derived from the arithmetic, not measured:
  * 16-bit outputs: <= 1 ulp (the lemma: the kernel's fp32 value is within
    2^-11 relative of the oracle's before the RNE cast, fast forms included);
  * fp32 outputs: the CUDA math library's documented maximum error plus one ulp
    for the oracle's own rounding of its double result (reading R12):
    expf 2, logf 1, tanhf 2 ulp; sigmoid = 1/(1 + expf(-v)) 2 + 1 + 1; GELU-erf
    = v * normcdff(v), normcdff 5 ulp, + 1 for the product (below v = -13.2
    normcdff's result is subnormal: 4 |v| 2^-149 absolute).  GELU-tanh keeps its
    MUFU form for fp32 outputs too: relative error <= (12 + 3|a|) u with
    a = v (C2 + C1 v^2) the log2-domain argument (ex2.approx 2^-22, rcp.approx,
    three roundings, and the fp32 rounding of a amplified by ln2 |a|), plus
    16 * 2^-126 absolute: ex2/rcp.approx.ftz flush subnormal intermediates;
  * division by a loop-invariant divisor (the packed Markstein form) and every
    IEEE operation: bit-exact, special operands included.
"""
import numpy as np
import pytest
import torch

from oracle import oracle as O

from harness import assert_bitexact, assert_ulp, check_rowstats, ordered32, run_gpu

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

F32 = np.float32
SPECIAL = [0.0, -0.0, np.inf, -np.inf, np.nan, 65504.0, -65504.0, 1e-7, -1e-7, 6e-8, 3e38, -3e38, 1e-40]


def _inputs(n, lo, hi, seed, dtype):
    v = np.concatenate([np.random.default_rng(seed).uniform(lo, hi, n - len(SPECIAL)), SPECIAL]).astype(F32)
    return v.astype(np.float16) if dtype == "f16" else v


def _ew(expr, n, in_dtype, out_dtype, extra=None):
    d = {"name": "t", "loops": {"r": 8, "i": n // 8},
         "tensors": {"a": {"shape": [8, n // 8], "dtype": in_dtype, "role": "in", "init": None, "strides": None},
                     "out": {"shape": [8, n // 8], "dtype": out_dtype, "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "assign", "loops": ["r", "i"], "write": ("out", ["r", "i"]),
                    "reads": [("a", ["r", "i"])], "expr": expr}]}
    if extra:
        extra(d)
    return d


F32_ULP = {"exp": 3, "log": 2, "tanh": 3, "sigmoid": 5, "gelu_erf": 7}


@pytest.mark.parametrize("op", ["exp", "log", "tanh", "sigmoid", "gelu_tanh", "gelu_erf"])
@pytest.mark.parametrize("out_dtype", ["f16", "bf16", "f32"])
def test_transcendental_sweep_and_special_values(op, out_dtype):
    n = 8 * 4096
    lo, hi = {"exp": (-20, 12), "log": (-1, 70000), "tanh": (-12, 12), "sigmoid": (-30, 30),
              "gelu_tanh": (-14, 10), "gelu_erf": (-14, 10)}[op]
    for in_dtype in ("f32", "f16"):
        x = _inputs(n, lo, hi, 7, in_dtype)
        d = _ew([("load", 0), (op, 0)], n, in_dtype, out_dtype)
        got, _ = run_gpu(d, {"a": x})
        ref = O.run(d, {"a": x})["out"]
        if out_dtype != "f32":
            assert_ulp(got["out"], ref, 1, f"{op} {in_dtype}->{out_dtype}")
        elif op == "gelu_tanh":
            v = x.astype(np.float64)
            c2 = -2.0 * 0.7978845608028654 * 1.4426950408889634
            a = np.abs(v * (c2 + 0.044715 * c2 * v * v))
            g, r = got["out"].astype(np.float64), ref.astype(np.float64)
            fin = np.isfinite(r)
            assert np.array_equal(np.isnan(got["out"]), np.isnan(ref))
            assert np.array_equal(g[~fin & ~np.isnan(r)], r[~fin & ~np.isnan(r)])
            tol = (12 + 3 * a[fin]) * 2.0 ** -24 * np.abs(r[fin]) + 16 * 2.0 ** -126   # MUFU forms flush subnormals
            assert np.all(np.abs(g[fin] - r[fin]) <= tol), np.max(np.abs(g[fin] - r[fin]) / tol)
        elif op == "gelu_erf":
            # v * normcdff(v): where Phi(v) < 2^-126 (v < -13.2) normcdff returns a subnormal, whose
            # absolute error (a few units of 2^-149) the product scales by |v|
            g, r = got["out"], ref
            d = np.abs(ordered32(g) - ordered32(r))
            nan = np.isnan(g) & np.isnan(r)
            sub = np.abs(g.astype(np.float64) - r.astype(np.float64)) <= 4 * np.abs(x.astype(np.float64)) * 2.0 ** -149
            bad = ~nan & (d > F32_ULP[op]) & ~sub
            assert not bad.any(), (x[bad][:4], g[bad][:4], r[bad][:4])
        else:
            assert_ulp(got["out"], ref, F32_ULP[op], f"{op} {in_dtype}->f32")


def test_gelu_tanh_f16_output_dense_sweep_including_the_subnormal_band():
    """Every f16 value in [-12, 8] (the band v in [-9, -4] has f16-subnormal GELU
    outputs) plus +-0, +-inf, NaN and |v| up to 65504."""
    h = np.arange(0, 0x10000, dtype=np.uint32).astype(np.uint16).view(np.float16)
    v = h[(np.abs(h.astype(F32)) <= 12) | ~np.isfinite(h) | (np.abs(h.astype(F32)) >= 60000)]
    n = (len(v) + 7) // 8 * 8
    x = np.concatenate([v, np.zeros(n - len(v), np.float16)])
    d = _ew([("load", 0), ("gelu_tanh", 0)], n, "f16", "f16")
    got, _ = run_gpu(d, {"a": x})
    assert_ulp(got["out"], O.run(d, {"a": x})["out"], 1, "gelu f16")


def test_cfg4a_gelu_special_values_through_the_row_kernel():
    """cfg4a's fused kernel (bias + GELU + row mean/var) on rows holding +-0,
    +-inf, NaN, +-65504 and a sweep of [-12, 8]: y within 1 ulp, statistics
    normwise (R16), non-finite statistics where the oracle has them."""
    import workloads as W
    B, S, H = 2, 24, 768
    d = W.cfg4a(B, S, H)
    x = W.make_inputs(d)
    rows = x["x"].reshape(B * S, H)
    rows[0] = np.linspace(-12, 8, H).astype(np.float16)
    rows[1] = np.linspace(-9, -4, H).astype(np.float16)                    # f16-subnormal GELU outputs
    rows[2, :6] = [0.0, -0.0, 65504, -65504, 1000, -1000]
    rows[3, 5] = np.inf
    rows[4, 7] = -np.inf
    rows[5, 100] = np.nan
    rows[6, :] = -np.inf
    x["bias"][:] = 0
    got, op = run_gpu(d, x)
    assert op.info()["launches"][0]["class"] == "row_reduce"
    check_rowstats(d, x, got)


# ---------------------------------------------------------------- division
@pytest.mark.parametrize("out_dtype", ["f16", "bf16", "f32"])
@pytest.mark.parametrize("offset", [0, 1])
def test_division_by_invariant_is_ieee_on_special_values(out_dtype, offset):
    """x / c and x / d[r] (a per-row divisor: invariant along the vector loop) with
    16-bit outputs take the packed Markstein form; every lane must equal IEEE
    division — inf/0, x/0, x/inf, overflowing and underflowing quotients, NaN,
    subnormal and huge divisors — on aligned and misaligned (scalar) variants."""
    n = 8 * 2048
    x = _inputs(n, -70000, 70000, 11, "f32")
    x[::97] = np.float32(3e38)
    x[1::89] = np.float32(1e-38)
    divs = np.array([3.0, -0.0, 0.0, np.inf, -np.inf, np.nan, 1e-40, 3e38, 0.1], F32)

    def per_row(d):
        d["tensors"]["dv"] = {"shape": [8], "dtype": "f32", "role": "in", "init": None, "strides": None}
        d["stmts"][0]["reads"].append(("dv", ["r"]))
    for c in (3.0, 0.1, 7e-39, 1e30, -2.5):
        d = _ew([("load", 0), ("const", c), ("div", 0, 1)], n, "f32", out_dtype)
        got, _ = run_gpu(d, {"a": x}, offset=offset)
        assert_bitexact(got["out"], O.run(d, {"a": x})["out"], f"x/{c}")
    for k in range(0, len(divs), 8):
        dv = np.resize(divs[k:k + 8], 8).astype(F32)
        d = _ew([("load", 0), ("load", 1), ("div", 0, 1)], n, "f32", out_dtype, per_row)
        got, _ = run_gpu(d, {"a": x, "dv": dv}, offset=offset)
        assert_bitexact(got["out"], O.run(d, {"a": x, "dv": dv})["out"], f"x/d[r] {dv}")


def test_division_then_cancellation_is_still_exact():
    """-x/1.5 + y with an f16 output (fuzz seed 21's case): the quotient feeds an add."""
    n = 8 * 1024
    rng = np.random.default_rng(21)
    a = rng.uniform(-4, 4, n).astype(F32)

    def two(d):
        d["tensors"]["b"] = {"shape": [8, n // 8], "dtype": "f32", "role": "in", "init": None, "strides": None}
        d["stmts"][0]["reads"].append(("b", ["r", "i"]))
    d = _ew([("load", 0), ("neg", 0), ("const", -1.5), ("div", 1, 2), ("load", 1), ("add", 3, 4)], n, "f32", "f16",
            two)
    b = (-(-a / F32(-1.5)) + rng.uniform(-1e-3, 1e-3, n).astype(F32)).astype(F32)
    got, _ = run_gpu(d, {"a": a, "b": b})
    assert_bitexact(got["out"], O.run(d, {"a": a, "b": b})["out"], "cancel")


# ---------------------------------------------------------------- max / min (R24)
def test_max_min_nan_and_signed_zero_on_gpu():
    n = 8 * 64
    P, N, Q = 0.0, -0.0, np.nan
    pa = np.array([P, N, N, P, Q, 1.0, Q, N, -2.0, np.inf, -np.inf], F32)
    pb = np.array([N, P, N, P, 1.0, Q, Q, -1.0, N, Q, 3.0], F32)
    a = np.resize(pa, n).astype(F32)
    b = np.resize(pb, n).astype(F32)

    def two(d):
        d["tensors"]["b"] = {"shape": [8, n // 8], "dtype": "f32", "role": "in", "init": None, "strides": None}
        d["stmts"][0]["reads"].append(("b", ["r", "i"]))
    for op in ("max", "min"):
        for out in ("f32", "f16"):
            d = _ew([("load", 0), ("load", 1), (op, 0, 1)], n, "f32", out, two)
            got, _ = run_gpu(d, {"a": a, "b": b})
            assert_bitexact(got["out"], O.run(d, {"a": a, "b": b})["out"], f"{op}->{out}")
