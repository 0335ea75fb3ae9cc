"""Pins of the C oracle against things other than itself (CPU only).

Every pin is either a library routine computing the same definition (numpy /
torch, which share no code with the oracle), a closed form, an invariant of
the paper's semantics, or brute force on a tiny case.  SURVEY §8(c) "What pins
each part" lists them; DESIGN.md §3 maps each pin to the oracle function.
"""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import oracle as O


def _eq_bits_nan(a, b):
    a = np.asarray(a)
    b = np.asarray(b)
    if a.dtype.kind == "f":
        both_nan = np.isnan(a.astype(np.float32)) & np.isnan(b.astype(np.float32))
        return np.all((a.view(np.uint16 if a.itemsize == 2 else np.uint32) ==
                       b.view(np.uint16 if b.itemsize == 2 else np.uint32)) | both_nan)
    return np.array_equal(a, b)


# --------------------------------------------------------------------------
# element conversions (IEEE binary16 / bfloat16) vs numpy / torch

def test_f16_decode_all_patterns():
    h = np.arange(65536, dtype=np.uint32).astype(np.uint16)
    ref = h.view(np.float16).astype(np.float32)
    got = np.array([O.f16_bits_to_f32(int(x)) for x in h], np.float32)
    assert _eq_bits_nan(got, ref)


def test_f16_encode_vs_numpy():
    rng = np.random.default_rng(0)
    vals = np.concatenate([
        rng.standard_normal(20000).astype(np.float32) * 10,
        rng.uniform(-70000, 70000, 5000).astype(np.float32),
        (rng.uniform(-1, 1, 5000) * 2.0 ** -14).astype(np.float32),   # subnormal range
        (rng.uniform(-1, 1, 2000) * 2.0 ** -24).astype(np.float32),   # round-to-zero edge
        np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 65504, 65519.99, 65520, 65536,
                  2.0 ** -24, 2.0 ** -25, 3 * 2.0 ** -26, 2.0 ** -14, 1e-45, 3.4e38],
                 np.float32),
    ])
    # exact halfway cases between consecutive halves
    h = np.arange(0, 0x7BFF, 7, dtype=np.uint16)
    lo = h.view(np.float16).astype(np.float64)
    hi = (h + 1).view(np.float16).astype(np.float64)
    vals = np.concatenate([vals, ((lo + hi) / 2).astype(np.float32)])
    ref = vals.astype(np.float16).view(np.uint16)
    got = np.array([O.f32_to_f16_bits(float(v)) for v in vals], np.uint16)
    nan = np.isnan(vals)
    assert np.array_equal(got[~nan], ref[~nan])
    assert np.all((got[nan] & 0x7C00) == 0x7C00) and np.all((got[nan] & 0x3FF) != 0)


def test_bf16_vs_torch():
    L = O.lib()
    rng = np.random.default_rng(1)
    vals = np.concatenate([rng.standard_normal(20000).astype(np.float32) * 100,
                           np.array([0, -0.0, np.inf, -np.inf, 3.4e38, 1e-40], np.float32)])
    ref = torch.from_numpy(vals).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    got = np.array([L.orc_f32_to_bf16(float(v)) for v in vals], np.uint16)
    assert np.array_equal(got, ref)


# --------------------------------------------------------------------------
# cfg1: elementwise with broadcast

def test_cfg1_tiny_brute_force_vs_numpy():
    d = W.cfg1()
    x = W.make_inputs(d)
    out = O.run(d, x)["out"].reshape(4, 8, 16)
    ref = np.maximum((x["x"].reshape(4, 8, 16) + x["bias"]) * x["y"].reshape(4, 8, 16),
                     np.float32(0))
    assert np.array_equal(out.view(np.uint32), (ref + np.float32(0)).view(np.uint32))
    # a few hand-evaluated points (brute force, one element at a time)
    for (a, b, c) in [(0, 0, 0), (3, 7, 15), (1, 4, 9)]:
        xv = x["x"][a * 128 + b * 16 + c]
        yv = x["y"][a * 128 + b * 16 + c]
        v = np.float32(np.float32(xv + x["bias"][c]) * yv)
        assert out[a, b, c] == (v if v > 0 else np.float32(0))


def test_cfg1_broadcast_equals_explicit_tiling():
    """Broadcast access bias[c] == the same op on a materialised [A,B,C] bias."""
    d = W.cfg1(4, 8, 16)
    x = W.make_inputs(d)
    ref = O.run(d, x)["out"]
    d2 = W.cfg1(4, 8, 16)
    d2["tensors"]["bias"] = {"shape": [4, 8, 16], "dtype": "f32", "role": "in",
                             "init": None, "strides": None}
    d2["stmts"][0]["reads"][1] = ("bias", ["a", "b", "c"])
    x2 = dict(x)
    x2["bias"] = np.tile(x["bias"], 32)
    assert np.array_equal(O.run(d2, x2)["out"].view(np.uint32), ref.view(np.uint32))
    # and expand-style stride-0 tensor dims give the same bits (R20 case iii)
    d3 = W.cfg1(4, 8, 16)
    d3["tensors"]["bias"] = {"shape": [4, 8, 16], "dtype": "f32", "role": "in",
                             "init": None, "strides": [0, 0, 1]}
    d3["stmts"][0]["reads"][1] = ("bias", ["a", "b", "c"])
    assert np.array_equal(O.run(d3, x)["out"].view(np.uint32), ref.view(np.uint32))


def test_relu_signed_zero_and_nan():
    d = W.cfg1(1, 1, 4)
    x = {"x": np.array([-0.0, np.nan, -1.0, 2.0], np.float32),
         "y": np.ones(4, np.float32), "bias": np.zeros(4, np.float32)}
    out = O.run(d, x)["out"]
    assert out.view(np.uint32).tolist()[:3] == [0, 0, 0]  # +0 for -0, NaN, negatives (R15)
    assert out[3] == 2.0


# --------------------------------------------------------------------------
# cfg2: BN inference + ReLU + cast

def test_cfg2_vs_numpy_float32_same_order():
    d = W.cfg2(N=2, C=8, H=12, W=20)
    x = W.make_inputs(d)
    y = O.run(d, x)["y"].reshape(2, 8, 12, 20)
    scale = x["gamma"] / np.sqrt(x["var"] + np.float32(1e-5))
    shift = x["beta"] - x["mean"] * scale
    v = x["x"].reshape(2, 8, 12, 20) * scale[None, :, None, None] + shift[None, :, None, None]
    ref = np.where(v > 0, v, np.float32(0)).astype(np.float16)
    assert np.array_equal(y.view(np.uint16), ref.view(np.uint16))


def test_cfg2_identity_bn_is_relu_cast():
    d = W.cfg2(N=2, C=4, H=8, W=8, eps=0.0)
    x = W.make_inputs(d)
    x["gamma"][:] = 1
    x["var"][:] = 1
    x["beta"][:] = 0
    x["mean"][:] = 0
    y = O.run(d, x)["y"]
    ref = np.maximum(x["x"], np.float32(0)).astype(np.float16)
    assert np.array_equal(y.view(np.uint16), (ref + np.float16(0)).view(np.uint16))


# --------------------------------------------------------------------------
# cfg3: NCHW -> NHWC transpose * s

def _nhwc_to_nchw(N, C, H, Wd, s, dtype="f16"):
    d = W.cfg3(N, C, H, Wd, s, dtype)
    d["tensors"]["x"]["shape"] = [N, H, Wd, C]
    d["tensors"]["out"]["shape"] = [N, C, H, Wd]
    d["stmts"][0]["write"] = ("out", ["n", "c", "h", "w"])
    d["stmts"][0]["reads"] = [("x", ["n", "h", "w", "c"])]
    return d


def test_cfg3_transpose_roundtrip_identity():
    N, C, H, Wd = 2, 24, 5, 7
    d = W.cfg3(N, C, H, Wd, s=1.0)
    d["tensors"]["x"]["init"] = ("special", 9)
    x = W.make_inputs(d)
    t = O.run(d, x)["out"]
    back = O.run(_nhwc_to_nchw(N, C, H, Wd, 1.0), {"x": t})["out"]
    assert _eq_bits_nan(back, x["x"])
    # s = 2 then s = 0.5 is the identity as long as nothing overflows
    d2 = W.cfg3(N, C, H, Wd, s=2.0)
    x2 = W.make_inputs(d2)
    t2 = O.run(d2, x2)["out"]
    back2 = O.run(_nhwc_to_nchw(N, C, H, Wd, 0.5), {"x": t2})["out"]
    assert _eq_bits_nan(back2, x2["x"])


def test_cfg3_vs_numpy_permute():
    N, C, H, Wd = 2, 16, 6, 10
    d = W.cfg3(N, C, H, Wd, s=0.5)
    d["tensors"]["x"]["init"] = ("special", 9)
    x = W.make_inputs(d)
    out = O.run(d, x)["out"]
    ref = (x["x"].reshape(N, C, H, Wd).transpose(0, 2, 3, 1).astype(np.float32) *
           np.float32(0.5)).astype(np.float16).reshape(-1)
    assert _eq_bits_nan(out, ref)


# --------------------------------------------------------------------------
# cfg4a: bias + GELU, row mean / var

def _rowstats_only(B, S, H):
    d = W.cfg4a(B, S, H)
    d["stmts"][0]["expr"] = [("load", 0)]
    d["stmts"][0]["reads"] = [("x", ["b", "s", "h"])]
    return d


def test_row_sum_of_ones_and_constant_rows():
    d = _rowstats_only(2, 3, 768)
    x = {"x": np.ones(2 * 3 * 768, np.float16), "bias": np.zeros(768, np.float16)}
    r = O.run(d, x)
    assert np.all(r["mean"] == 1.0) and np.all(r["var"] == 0.0)
    x["x"][:] = np.float16(-2.5)
    r = O.run(d, x)
    assert np.all(r["mean"] == -2.5) and np.all(r["var"] == 0.0)


def test_row_arange_closed_form():
    d = _rowstats_only(1, 2, 768)
    row = np.arange(768, dtype=np.float16)
    x = {"x": np.concatenate([row, row]), "bias": np.zeros(768, np.float16)}
    r = O.run(d, x)
    assert np.all(r["mean"] == np.float32(383.5))
    assert np.all(r["var"] == np.float32((768 ** 2 - 1) / 12))


def _ordered(f32):
    """Map fp32 bit patterns to integers whose differences count ulps."""
    i = f32.view(np.int32).astype(np.int64)
    return np.where(i < 0, -(i & 0x7FFFFFFF), i)


def _gelu_decimal(v):
    """GELU-tanh in 60-digit decimal arithmetic (independent reference)."""
    from decimal import Decimal, getcontext
    getcontext().prec = 60
    d = Decimal(float(v))
    pi = Decimal("3.14159265358979323846264338327950288419716939937510582097494")
    u = (Decimal(2) / pi).sqrt() * (d + Decimal("0.044715") * d * d * d)
    e = (2 * u).exp()
    return float(Decimal("0.5") * d * (2 * e / (e + 1)))     # 1 + tanh u = 2e/(e+1)


def test_gelu_tanh_vs_torch_decimal_and_identities():
    L = O.lib()
    v = np.concatenate([np.linspace(-5, 8, 3001), [0.0, 1e-3, -1e-3, 30]]).astype(np.float32)
    got = np.array([L.orc_gelu_tanh(float(a)) for a in v], np.float32)
    ref = torch.nn.functional.gelu(torch.from_numpy(v.astype(np.float64)),
                                   approximate="tanh").numpy().astype(np.float32)
    assert np.abs(_ordered(got) - _ordered(ref)).max() <= 1
    # deep negative tail, where 1 + tanh(u) cancels in double: 60-digit reference
    tail = np.linspace(-12, -5, 57).astype(np.float32)
    got_t = np.array([L.orc_gelu_tanh(float(a)) for a in tail], np.float32)
    ref_t = np.array([_gelu_decimal(a) for a in tail]).astype(np.float32)
    assert np.abs(_ordered(got_t) - _ordered(ref_t)).max() <= 1
    assert L.orc_gelu_tanh(0.0) == 0.0
    # gelu(v) - gelu(-v) = v (odd inner argument of tanh), up to rounding
    gm = np.array([L.orc_gelu_tanh(float(-a)) for a in v], np.float32)
    assert np.allclose(got.astype(np.float64) - gm, v, rtol=0, atol=4e-7 * np.maximum(1, np.abs(v)))


def test_cfg4a_vs_torch_var_mean():
    d = W.cfg4a(2, 16, 768)
    x = W.make_inputs(d)
    r = O.run(d, x)
    xv = torch.from_numpy(x["x"].astype(np.float64).reshape(2, 16, 768))
    bv = torch.from_numpy(x["bias"].astype(np.float64))
    y_ref = torch.nn.functional.gelu((xv.float() + bv.float()).double(), approximate="tanh")
    y_ref = y_ref.float().half()
    y = r["y"].reshape(2, 16, 768)
    # y: oracle rounds the double GELU once to fp32 then to fp16
    diff = np.abs(y.astype(np.float32) - y_ref.float().numpy())
    ulp16 = np.spacing(np.abs(y_ref.float().numpy()).astype(np.float16)).astype(np.float32)
    assert np.all(diff <= ulp16)
    var, mean = torch.var_mean(torch.from_numpy(y.astype(np.float64)), dim=-1, unbiased=False)
    assert np.allclose(r["mean"].reshape(2, 16), mean.numpy(), rtol=1e-6, atol=1e-7)
    assert np.allclose(r["var"].reshape(2, 16), var.numpy(), rtol=1e-6, atol=1e-7)


# --------------------------------------------------------------------------
# cfg4b: column sum

def test_colsum_of_ones_equals_extent():
    d = W.cfg4b(65536, 8, init=("ones",))
    r = O.run(d, W.make_inputs(d))
    assert np.all(r["out"] == 65536.0)


def test_colsum_powers_of_two_exact_and_vs_numpy():
    R, Cn = 1000, 16
    d = W.cfg4b(R, Cn)
    x = W.make_inputs(d)
    x["x"] = np.tile((2.0 ** (np.arange(Cn) % 8 - 4)).astype(np.float16), R)
    r = O.run(d, x)
    assert np.array_equal(r["out"], (R * 2.0 ** (np.arange(Cn) % 8 - 4)).astype(np.float32))
    d = W.cfg4b(3000, 40)
    x = W.make_inputs(d)
    r = O.run(d, x)
    ref = x["x"].astype(np.float64).reshape(3000, 40).sum(0)
    assert np.allclose(r["out"], ref, rtol=1e-6, atol=1e-6)


def test_reduce_max_and_finalize():
    d = W.cfg4b(50, 6)
    d["stmts"][0]["op"] = "max"
    d["stmts"][0]["finalize"] = [("acc",), ("const", 2.0), ("mul", 0, 1)]
    x = W.make_inputs(d)
    r = O.run(d, x)
    ref = x["x"].astype(np.float32).reshape(50, 6).max(0) * 2
    assert np.array_equal(r["out"], ref)


# --------------------------------------------------------------------------
# Fig. 2: schedule equivalence of the running example

def test_fig2_orders_a_and_c_identical_and_vs_numpy():
    N = 12
    da = W.fig2_running_example(N, order_y=("i", "j", "k"))   # Fig. 2(a) order
    dc = W.fig2_running_example(N, order_y=("i", "k", "j"))   # Fig. 2(c) order
    x = W.make_inputs(da)
    ra = O.run(da, x)
    rc = O.run(dc, x)
    assert np.array_equal(ra["C"], rc["C"]) and np.array_equal(ra["B"], rc["B"])
    A = x["A"].reshape(N, N).astype(np.float64)
    D = x["D"].reshape(N, N, N).astype(np.float64)
    Bm = A + 1
    Cm = x["C"].reshape(N, N).astype(np.float64) + np.einsum("ik,kij->ij", Bm, D)
    assert np.array_equal(ra["C"].reshape(N, N), Cm.astype(np.float32))
    assert np.array_equal(ra["B"].reshape(N, N), Bm.astype(np.float32))


def test_validation_rejects_out_of_bounds():
    d = W.cfg1()
    d["stmts"][0]["reads"][1] = ("bias", [("c", 1)])  # bias[c+1] overruns
    with pytest.raises(ValueError):
        O.run(d, W.make_inputs(d))
