"""Edge cases: empty domains and index spans beyond 2^31 elements.

Empty: a box domain 0 <= i < N with N = 0 has no statement
instance, so the statement writes nothing (reading R28) — the plan has no
launch for it and running it is a no-op.

Large: spans past 2^31 elements switch the generated kernels to 64-bit index
arithmetic.  Inputs there are a deterministic index pattern, filled on the
device in chunks and re-created on the host for the sampled slices the
oracle checks (or checked against a closed form), so no 9 GB host copy is
needed.
"""
import numpy as np
import pytest

import workloads as W
from oracle import oracle as O

from harness import assert_bitexact, assert_normwise, assert_ulp, abs_terms_desc


def fop():
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    return FusedOp


def two_statements(A, B):
    """out1[a] = 2*x[a] over a;  out2[b] = y[b] + 1 over b (independent loops)."""
    return {"name": "two_statements", "loops": {"a": A, "b": B},
            "tensors": {"x": {"shape": [A], "dtype": "f32", "role": "in", "init": ("normal", 0.0, 1.0, 71)},
                        "y": {"shape": [B], "dtype": "f32", "role": "in", "init": ("normal", 0.0, 1.0, 72)},
                        "out1": {"shape": [A], "dtype": "f32", "role": "out"},
                        "out2": {"shape": [B], "dtype": "f32", "role": "out"}},
            "stmts": [{"kind": "assign", "loops": ["a"], "write": ("out1", ["a"]), "reads": [("x", ["a"])],
                       "expr": [("load", 0), ("const", 2.0), ("mul", 0, 1)]},
                      {"kind": "assign", "loops": ["b"], "write": ("out2", ["b"]), "reads": [("y", ["b"])],
                       "expr": [("load", 0), ("const", 1.0), ("add", 0, 1)]}]}


EMPTY = {
    "cfg2_N0": lambda: W.cfg2(N=0, C=8, H=4, W=4),
    "cfg3_N0": lambda: W.cfg3(N=0, C=16, H=3, W=5),
    "cfg4a_B0": lambda: W.cfg4a(B=0, S=4, H=64),
    "cfg4b_R0": lambda: W.cfg4b(R=0, C=64),
    "scan_T1": lambda: W.N3["scan_time"](B=2, T=1, H=8),   # time loop of extent T-1 = 0
}


# ------------------------------------------------------------ empty domains (CPU)
@pytest.mark.parametrize("name", list(EMPTY))
def test_empty_domain_plans_no_launch(name):
    d = EMPTY[name]()
    op = fop()(d, jit=0)
    assert op.info()["launches"] == []


@pytest.mark.parametrize("name", list(EMPTY))
def test_oracle_empty_domain_writes_nothing(name):
    d = EMPTY[name]()
    x = W.make_inputs(d)
    outs = W.alloc_outputs(d)   # NaN pattern: nothing may overwrite it
    ref = O.run(d, x, outputs={n: b.copy() for n, b in outs.items()})
    for n, t in d["tensors"].items():
        k = W.tensor_span(t)
        if t["role"] == "out":
            assert np.array_equal(ref[n][:k].view(np.uint8), outs[n][:k].view(np.uint8)), n
        elif t["role"] == "inout":
            assert np.array_equal(ref[n][:k].view(np.uint8), x[n][:k].view(np.uint8)), n


def test_mixed_empty_and_nonempty_statements_plan():
    op = fop()(two_statements(0, 100), jit=0)
    li = op.info()["launches"]
    assert len(li) == 1 and li[0]["stmts"] == [1]


# ------------------------------------------------------------ empty domains (GPU)
@pytest.mark.gpu
@pytest.mark.parametrize("name", list(EMPTY))
def test_empty_domain_run_is_noop(name):
    from harness import run_gpu
    d = EMPTY[name]()
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)                      # outputs start as the NaN pattern
    ref = O.run(d, x, outputs=W.alloc_outputs(d))
    for n in got:
        assert_bitexact(got[n], ref[n], n)


@pytest.mark.gpu
def test_mixed_empty_and_nonempty_statements_run():
    from harness import run_gpu
    d = two_statements(0, 1000)
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    assert_bitexact(got["out2"], O.run(d, x)["out2"], "out2")


# ------------------------------------------------------------ > 2^31 elements (GPU)
def pattern_host(start, n, dtype, mod=251, scale=1.0 / 32):
    """((i mod 251) - 125) / 32 for global element i in [start, start + n): exact in f16/bf16/f32."""
    idx = np.arange(start, start + n, dtype=np.int64)
    v = ((idx % mod) - mod // 2).astype(np.float32) * np.float32(scale)
    return v.astype(W.NP_DTYPE[dtype]) if dtype != "bf16" else None


def fill_pattern(t, mod=251, scale=1.0 / 32):
    import torch
    flat = t.view(-1)
    step = 1 << 26
    for s in range(0, flat.numel(), step):
        e = min(flat.numel(), s + step)
        idx = torch.arange(s, e, device=t.device, dtype=torch.int64)
        flat[s:e] = (((idx % mod) - mod // 2).to(torch.float32) * scale).to(t.dtype)


def _dev(desc, name):
    import torch
    from harness import TORCH_DT
    t = desc["tensors"][name]
    return torch.empty(W.tensor_span(t), dtype=TORCH_DT[t["dtype"]], device="cuda")


def _free():
    import gc
    import torch
    gc.collect()
    torch.cuda.empty_cache()


@pytest.mark.gpu
def test_ew_bn_past_2p31_elements():
    from harness import to_device, to_host
    N = 2720                                    # 2720 x 64 x 112 x 112 = 2.18e9 elements
    d = W.cfg2(N=N)
    op = fop()(d)
    assert "typedef unsigned long long idx_t" in op.source(0)
    small = W.make_inputs(W.cfg2(N=1))          # the [64] parameters do not depend on N
    dev = {n: to_device(small[n], "f32") for n in ("gamma", "beta", "mean", "var")}
    dev["x"] = _dev(d, "x")
    dev["y"] = _dev(d, "y")
    fill_pattern(dev["x"])
    op.run(dev)
    per = 64 * 112 * 112
    for n in (0, N // 2 + 1, N - 1):
        d1 = W.cfg2(N=1)
        xs = dict(small)
        xs["x"] = pattern_host(n * per, per, "f32")
        ref = O.run(d1, xs)["y"]
        assert_bitexact(to_host(dev["y"][n * per:(n + 1) * per], "f16"), ref, f"y n={n}")
    del dev
    _free()


@pytest.mark.gpu
def test_transpose_past_2p31_elements():
    from harness import to_host
    N = 2720                                    # 2720 x 256 x 56 x 56 = 2.18e9 elements
    d = W.cfg3(N=N)
    op = fop()(d)
    assert "typedef unsigned long long idx_t" in op.source(0)
    dev = {"x": _dev(d, "x"), "out": _dev(d, "out")}
    fill_pattern(dev["x"])
    op.run(dev)
    per = 256 * 56 * 56
    for n in (0, N // 2 + 1, N - 1):
        d1 = W.cfg3(N=1)
        ref = O.run(d1, {"x": pattern_host(n * per, per, "f16")})["out"]
        assert_bitexact(to_host(dev["out"][n * per:(n + 1) * per], "f16"), ref, f"out n={n}")
    del dev
    _free()


@pytest.mark.gpu
def test_row_reduce_past_2p31_elements():
    from harness import to_device, to_host
    B = 5600                                    # 5600 x 512 x 768 = 2.2e9 elements
    d = W.cfg4a(B=B)
    op = fop()(d)
    assert "typedef unsigned long long idx_t" in op.source(0)
    small = W.make_inputs(W.cfg4a(B=1))
    dev = {"bias": to_device(small["bias"], "f16")}
    for n in ("x", "y", "mean", "var"):
        dev[n] = _dev(d, n)
    fill_pattern(dev["x"])
    op.run(dev)
    per = 512 * 768
    for b in (0, B // 2 + 1, B - 1):
        d1 = W.cfg4a(B=1)
        xs = {"x": pattern_host(b * per, per, "f16"), "bias": small["bias"]}
        ref = O.run(d1, xs)
        assert_ulp(to_host(dev["y"][b * per:(b + 1) * per], "f16"), ref["y"], 1, f"y b={b}")
        for name, si in (("mean", 1), ("var", 2)):
            got = to_host(dev[name][b * 512:(b + 1) * 512], "f32")
            scale = O.run(abs_terms_desc(d1, si), xs)[name]
            assert_normwise(got, ref[name], scale, 2e-3, f"{name} b={b}")
    del dev
    _free()


@pytest.mark.gpu
def test_colsum_past_2p31_elements_exact():
    """x[r][c] = ((c mod 7) - 3)/8 for every r: every partial sum is a multiple
    of 1/8 below 2^21, exact in fp32 in any order, so out[c] = R*x[0][c] exactly."""
    import torch
    from harness import to_host
    R = (1 << 21) + (1 << 17)                  # 2228224 x 1024 = 2.28e9 elements
    d = W.cfg4b(R=R)
    op = fop()(d)
    assert "typedef unsigned long long idx_t" in op.source(0)
    ws = torch.zeros(max(1, op.workspace_bytes), dtype=torch.uint8, device="cuda")
    x = _dev(d, "x").view(R, 1024)
    v = ((torch.arange(1024, device="cuda") % 7 - 3).to(torch.float32) / 8).to(torch.float16)
    x[:] = v
    out = _dev(d, "out")
    op.run({"x": x, "out": out}, workspace=ws)
    expect = (v.to(torch.float64) * R).to(torch.float32)
    assert_bitexact(to_host(out, "f32"), to_host(expect, "f32"), "out")
    del x, out, ws
    _free()
