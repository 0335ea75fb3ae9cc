"""fused operators shaped like the other Table I networks.

CPU: the oracle's evaluation of each new composition is pinned to torch
(float64 reference of the same formula, a library routine sharing no code with
the oracle).  GPU (marked): the CUDA path vs the oracle with the north_star
tolerances."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import oracle as O

SMALL = {
    "lstm_cell": dict(B=8, H=96),
    "mobilenet_bn_relu6": dict(N=2, C=24, H=14, W=14),
    "resnext_bn_add_relu": dict(N=2, C=32, H=7, W=8),
    "vgg_bias_relu": dict(N=2, C=16, H=9, W=16),
    "bert_layernorm": dict(B=2, S=16, H=768),
    "bert_softmax": dict(B=1, NH=3, S=128),
    # few long rows: several warps per row (ROW_REDUCE row_g > 1)
    "vocab_softmax": dict(R=5, V=4000),
    "wide_layernorm": dict(R=3, H=12288),
    # few vectors per row under long outer reduction loops: lanes split the outer iterations
    "bn_stats_nchw": dict(N=6, C=8, H=14, W=14),
    "bn_stats_small_hw": dict(N=64, C=8, H=4, W=4),     # 2 vectors per row: lanes split the samples
}


def _ulp16(a, b):
    from harness import ordered16
    return np.abs(ordered16(a) - ordered16(b))


def _assert_lstm(d, x, got, ref):
    """LSTM cell, fp32 outputs of transcendental compositions.  With u = 2^-24
    and the CUDA math library's documented bounds (expf, tanhf <= 2 ulp = 4u relative):
      sigmoid = 1/(1 + expf(-v)): <= 4u (expf, damped by e/(1+e)) + u (add) + u (rcp) = 6u;
      A = sigmoid(f) c_prev: 7u;  B = sigmoid(i) tanh(g): 6u + 4u + u = 11u;
      the oracle rounds each transcendental once (u) and each product (u): A 2u, B 3u;
      c = A + B: |gpu - ref| <= 9u|A| + 14u|B| + 2u|c| <= 16u (|A| + |B|)  (no absolute floor:
      the bound is normwise in the two products, which is where cancellation can hide);
      h = sigmoid(o) tanh(c) reads each side's OWN stored c, |d tanh| <= |dc|:
      |gpu - ref| <= 16u (|A| + |B|) + 16u |h| + 2^-149."""
    u = 2.0 ** -24
    B_, H = d["loops"]["b"], d["loops"]["h"]
    g = x["g"].astype(np.float64).reshape(B_, 4 * H)
    gi, gf, gg = g[:, :H], g[:, H:2 * H], g[:, 2 * H:3 * H]
    sig = lambda t: 1.0 / (1.0 + np.exp(-t))  # noqa: E731
    A = np.abs(sig(gf) * x["c_prev"].astype(np.float64).reshape(B_, H))
    Bm = np.abs(sig(gi) * np.tanh(gg))
    tol_c = (16 * u * (A + Bm)).reshape(-1)
    gc, rc = got["c"].astype(np.float64), ref["c"].astype(np.float64)
    assert np.all(np.abs(gc - rc) <= tol_c), float(np.max(np.abs(gc - rc) / tol_c))
    gh, rh = got["h_out"].astype(np.float64), ref["h_out"].astype(np.float64)
    tol_h = tol_c + 16 * u * np.abs(rh) + 2.0 ** -149
    assert np.all(np.abs(gh - rh) <= tol_h), float(np.max(np.abs(gh - rh) / tol_h))


def _assert_layernorm(d, x, got, ref):
    """y = t*gamma + beta with t = (x - mean)*rstd: mean and var are
    reductions (R16), so y may differ by 1 f16 ulp plus 1e-5 of the magnitudes
    entering the final add (|t*gamma| + |beta| + |gamma|), which bounds the
    statistics' error propagated through a cancelling add."""
    B, S, H = d["loops"]["b"], d["loops"]["s"], d["loops"]["h"]
    xx = x["x"].astype(np.float64).reshape(B * S, H)
    g = x["gamma"].astype(np.float64)
    b = x["beta"].astype(np.float64)
    mean = xx.mean(1, keepdims=True)
    t = (xx - mean) / np.sqrt(xx.var(1, keepdims=True) + 1e-12)
    scale = np.abs(t * g) + np.abs(b) + np.abs(g)
    gv = got.astype(np.float64).reshape(B * S, H)
    rv = ref.astype(np.float64).reshape(B * S, H)
    ulp = np.spacing(np.abs(ref.astype(np.float16))).astype(np.float64).reshape(B * S, H)
    err = np.abs(gv - rv)
    bad = err > ulp + 1e-5 * scale
    assert not bad.any(), (int(bad.sum()), float(err[bad].max()))


# ---------------------------------------------------------------- oracle pins (CPU)
def test_oracle_bn_stats_vs_torch():
    d = W.N4["bn_stats_nchw"](**SMALL["bn_stats_nchw"])
    x = W.make_inputs(d)
    r = O.run(d, x)
    xt = torch.from_numpy(x["x"].astype(np.float64).reshape(6, 8, 14, 14))
    var, mean = torch.var_mean(xt, dim=(0, 2, 3), unbiased=False)
    assert np.allclose(r["mean"], mean.numpy(), rtol=1e-6, atol=1e-7)
    # var from the f32-rounded mean (R17: later statements read stored values)
    m32 = torch.from_numpy(r["mean"].astype(np.float64)).view(1, 8, 1, 1)
    v2 = ((xt - m32) ** 2).mean(dim=(0, 2, 3))
    assert np.allclose(r["var"], v2.numpy(), rtol=1e-6, atol=0)
    assert np.allclose(r["var"], var.numpy(), rtol=1e-5, atol=0)


def test_bn_stats_row_geometry():
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    # 64 channel rows of 1568 vectors x 128 samples: clusters of 4 CTAs per row
    op = FusedOp(W.N4["bn_stats_nchw"](), autotune=0)
    (li,) = op.info()["launches"]
    assert li["class"] == "row_reduce" and li["vec_loop"] == "w" and li["grid"] == 256
    src = op.source(0)
    assert "__cluster_dims__(4, 1, 1)" in src and "fop::ld_dsmem" in src
    # 4x4 planes: 2 vectors per row under 64 samples -> lanes split the samples
    src = FusedOp(W.N4["bn_stats_nchw"](N=64, C=8, H=4, W=4), autotune=0).source(0)
    assert "ro_ = sub_;" in src and "vl_ < 2u" in src



def test_oracle_layernorm_vs_torch():
    d = W.N4["bert_layernorm"](**SMALL["bert_layernorm"])
    x = W.make_inputs(d)
    y = O.run(d, x)["y"]
    xt = torch.from_numpy(x["x"].astype(np.float64).reshape(2, 16, 768))
    ref = torch.nn.functional.layer_norm(xt, (768,), torch.from_numpy(x["gamma"].astype(np.float64)),
                                         torch.from_numpy(x["beta"].astype(np.float64)), eps=1e-12)
    assert _ulp16(y, ref.numpy().astype(np.float16).reshape(-1)).max() <= 1


def test_oracle_softmax_vs_torch():
    d = W.N4["bert_softmax"](**SMALL["bert_softmax"])
    x = W.make_inputs(d)
    y = O.run(d, x)["y"]
    ref = torch.softmax(torch.from_numpy(x["x"].astype(np.float64).reshape(1, 3, 128, 128)), -1)
    assert _ulp16(y, ref.numpy().astype(np.float16).reshape(-1)).max() <= 1
    assert np.allclose(y.astype(np.float64).reshape(-1, 128).sum(1), 1.0, atol=2e-2)


def test_oracle_vocab_softmax_vs_torch():
    d = W.N4["vocab_softmax"](R=3, V=1000)
    x = W.make_inputs(d)
    got = O.run(d, x)["y"].astype(np.float64).reshape(3, 1000)
    ref = torch.softmax(torch.from_numpy(x["x"].astype(np.float64).reshape(3, 1000)), dim=1).numpy()
    assert np.all(np.abs(got - ref) <= 2.0 ** -11 * np.abs(ref) + 2.0 ** -24)


def test_oracle_lstm_vs_torch():
    B, H = 8, 96
    d = W.N4["lstm_cell"](B, H)
    x = W.make_inputs(d)
    r = O.run(d, x)
    g = torch.from_numpy(x["g"].astype(np.float64).reshape(B, 4 * H))
    i, f, gg, o = g.split(H, dim=1)
    c = torch.sigmoid(f) * torch.from_numpy(x["c_prev"].astype(np.float64).reshape(B, H)) + \
        torch.sigmoid(i) * torch.tanh(gg)
    h = torch.sigmoid(o) * torch.tanh(torch.from_numpy(r["c"].astype(np.float64).reshape(B, H)))
    assert np.allclose(r["c"].reshape(B, H), c.numpy(), rtol=1e-6, atol=1e-6)
    assert np.allclose(r["h_out"].reshape(B, H), h.numpy(), rtol=1e-6, atol=1e-6)


def test_oracle_relu6_and_residual_vs_numpy():
    d = W.N4["mobilenet_bn_relu6"](**SMALL["mobilenet_bn_relu6"])
    x = W.make_inputs(d)
    y = O.run(d, x)["y"]
    sc = x["gamma"] / np.sqrt(x["var"] + np.float32(1e-5))
    sh = x["beta"] - x["mean"] * sc
    v = x["x"].astype(np.float32).reshape(2, 24, 14, 14) * sc[None, :, None, None] + sh[None, :, None, None]
    ref = np.minimum(np.maximum(v, np.float32(0)), np.float32(6)).astype(np.float16).reshape(-1)
    assert np.array_equal(y.view(np.uint16), (ref + np.float16(0)).view(np.uint16))
    d = W.N4["resnext_bn_add_relu"](**SMALL["resnext_bn_add_relu"])
    x = W.make_inputs(d)
    y = O.run(d, x)["y"]
    sc = x["gamma"] / np.sqrt(x["var"] + np.float32(1e-5))
    sh = x["beta"] - x["mean"] * sc
    v = (x["x"].astype(np.float32).reshape(2, 32, 7, 8) * sc[None, :, None, None] + sh[None, :, None, None]) + \
        x["res"].astype(np.float32).reshape(2, 32, 7, 8)
    ref = np.where(v > 0, v, np.float32(0)).astype(np.float16).reshape(-1)
    assert np.array_equal(y.view(np.uint16), ref.view(np.uint16))


# ---------------------------------------------------------------- GPU parity
@pytest.mark.gpu
@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("full", [False, True])
def test_n4_gpu_vs_oracle(name, full):
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from harness import run_gpu, assert_bitexact, assert_ulp
    d = W.N4[name]() if full else W.N4[name](**SMALL[name])
    if full and name in ("mobilenet_bn_relu6", "resnext_bn_add_relu", "vgg_bias_relu", "bert_softmax", "bert_layernorm"):
        loop = list(d["loops"])[0]
        d["loops"][loop] = 2                     # full per-sample shape, 2 samples (oracle time)
        for t in d["tensors"].values():
            if t["shape"] and t["shape"][0] == W.N4[name]()["loops"][loop] and len(t["shape"]) > 1:
                t["shape"][0] = 2
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert len(op.info()["launches"]) == 1
    ref = O.run(d, x)
    for n, v in got.items():
        if name == "lstm_cell":
            _assert_lstm(d, x, got, ref)
            break
        elif name in ("bert_layernorm", "wide_layernorm"):
            _assert_layernorm(d, x, v, ref[n])
        elif name in ("bert_softmax", "vocab_softmax"):
            assert_ulp(v, ref[n], 1, n)
        elif name.startswith("bn_stats"):
            from harness import abs_terms_desc, assert_normwise
            si = 0 if n == "mean" else 1
            assert_normwise(v, ref[n], O.run(abs_terms_desc(d, si), x)[n], 1e-5, n)
        else:
            assert_bitexact(v, ref[n], n)
