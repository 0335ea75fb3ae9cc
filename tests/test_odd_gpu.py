"""Odd innermost extents under a broadcast (round-2 cliff fix): no vector
width divides E[d_v] and a broadcast along d_v (bias[c]) keeps (c, r) from
collapsing, so the kernel flattens (c, r) into one loop of full-width vectors
and reads the broadcast access per element at c = flat index mod E[c]
(§V: vector and scalar accesses mixed in one statement).
Bit-exact against the oracle, aligned and misaligned, plus per-channel
BatchNorm on NHWC with an odd channel count (the scale/shift cone tabulated
over c and looked up per element)."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import oracle as O

from harness import assert_bitexact, run_gpu

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)


@pytest.mark.parametrize("R,C,dtype", [(1000, 1001, "f16"), (333, 13, "f32"), (64, 1001, "bf16"), (7, 9, "f16"),
                                       (5, 3, "f16"), (4099, 255, "f16")])
@pytest.mark.parametrize("offset", [0, 1])
def test_bias_add_over_odd_rows(R, C, dtype, offset):
    d = W.bias_add_rows(R, C, dtype)
    d["tensors"]["x"]["init"] = ("special", 63)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x, offset=offset)
    li = op.info()["launches"][0]
    if offset == 0 and C >= 8:
        assert li["width"] >= 4 and "PC_0" in op.source(), li      # flattened, full-width vectors
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("dims", [(2, 7, 9, 255), (3, 5, 5, 13), (1, 4, 4, 1001)])
def test_nhwc_bn_odd_channels(dims):
    d = W.cfg2_nhwc(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert_bitexact(got["y"], O.run(d, x)["y"], "y")


@pytest.mark.full_size
def test_bias_add_full_size_every_candidate():
    """[65536, 1001] f16 (a 1001-class classifier's logits over 65536 tokens), every tuning candidate."""
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    from harness import device_tensors, to_host
    d = W.bias_add_rows(65536, 1001, "f16")
    x = W.make_inputs(d)
    ref = O.run(d, x)["out"]
    nv = FusedOp(d).info()["launches"][0]["nvariants"]
    for k in range(nv):
        op = FusedOp(d, variant=k)
        dev = device_tensors(d, x)
        op.run(dev)
        torch.cuda.synchronize()
        assert_bitexact(to_host(dev["out"], "f16"), ref, f"candidate {k} {op.selected(0)[0]}")


@pytest.mark.parametrize("dims,dtype", [((2, 255, 56, 56), "f16"), ((1, 255, 7, 8), "f32"), ((2, 129, 4, 8), "bf16"),
                                        ((3, 33, 8, 8), "f16")])
@pytest.mark.parametrize("om", ["1", "0"])
def test_transpose_long_odd_channels_output_major_tile(monkeypatch, dims, dtype, om):
    """NCHW -> NHWC with a long odd C (255): the output rows carry no store vector, so a
    tile of whole NHWC rows is written flat; with the output-major tile (FOP_TR_SMEM_OM=1,
    the default for C >= 32) lanes scatter consecutive channels into the tile and read it
    out as 16 B vectors.  Both tile orientations bit-exact, NaN payloads of a pure move kept."""
    monkeypatch.setenv("FOP_TR_SMEM_OM", om)
    d = W.cfg3(*dims, dtype=dtype)
    d["tensors"]["x"]["init"] = ("special", 5)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.selected(0)[0].startswith("fop_transpose_smem")
    assert ("tw_" in op.source()) == (om == "1" and dims[1] >= 32)
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")
    d["stmts"][0]["expr"] = [("load", 0)]
    got, op = run_gpu(d, x)
    assert_bitexact(got["out"], O.run(d, x)["out"], "out (move)")


def _colred(R, C, dtype="f16", op="sum", expr=None):
    return {"name": "colred", "loops": {"r": R, "c": C},
            "tensors": {"x": {"shape": [R, C], "dtype": dtype, "role": "in", "init": ("normal", 0.0, 1.0, 71),
                              "strides": None},
                        "out": {"shape": [C], "dtype": "f32", "role": "out", "init": None, "strides": None}},
            "stmts": [{"kind": "reduce", "op": op, "loops": ["r", "c"], "write": ("out", ["c"]),
                       "reads": [("x", ["r", "c"])], "expr": expr or [("load", 0)]}]}


@pytest.mark.parametrize("R,C,dtype,op", [(65536, 1001, "f16", "sum"), (777, 1001, "f16", "sum"), (300, 13, "f16", "sum"),
                                          (5000, 37, "f32", "sum"), (2000, 257, "bf16", "sum"), (3001, 1001, "f16", "max"),
                                          (64, 9, "f16", "sum"), (4096, 1002, "f16", "sum"), (1000, 1004, "bf16", "max"),
                                          (8, 1001, "f16", "sum"), (40000, 3, "f16", "sum"), (6, 1001, "f32", "max")])
@pytest.mark.parametrize("offset", [0, 1])
@pytest.mark.parametrize("mode", ["fold", "shift", "shfl"])
def test_column_reduction_over_odd_rows(monkeypatch, R, C, dtype, op, offset, mode):
    """Column sums / maxima over rows of odd length, full-width vectors either way:
    fold (default when R >= P = W / gcd(C, W)): the first R - R mod P rows read as [R/P, P*C]
    with aligned vectors, the P*C wide-column sums folded into the C outputs by the last slab,
    which adds the R mod P remaining rows element-wise;
    shift: each row's window funnel-shifted out of two aligned 16 B chunks (the partial
    last vector's extra columns never stored); shfl: the second chunk shuffled from the
    neighbour lane.  Misaligned base pointers take the narrow variant."""
    import math
    from harness import abs_terms_desc, assert_normwise
    monkeypatch.setenv("FOP_COL_FOLD", "1" if mode == "fold" else "0")
    monkeypatch.setenv("FOP_COL_SHFL", "1" if mode == "shfl" else "0")
    d = _colred(R, C, dtype, op)
    x = W.make_inputs(d)
    got, o = run_gpu(d, x, offset=offset)
    if offset == 0:
        Wd = 16 // (4 if dtype == "f32" else 2)
        fold = mode == "fold" and R >= Wd // math.gcd(C, Wd)
        assert ("fold_flag" in o.source()) == fold, o.info()["launches"][0]
        assert ("__funnelshift_r" in o.source()) == (not fold and C >= Wd), o.info()["launches"][0]
    ref = O.run(d, x)["out"]
    if op == "max":
        assert_bitexact(got["out"], ref, "out")
    else:
        assert_normwise(got["out"], ref, O.run(abs_terms_desc(d, 0), x)["out"], 1e-5, "out")


@pytest.mark.full_size
def test_column_sum_of_squares_odd_rows_every_candidate():
    from harness import abs_terms_desc, assert_normwise, device_tensors, to_host
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    d = _colred(65536, 1001, "f16", "sum", [("load", 0), ("mul", 0, 0)])
    x = W.make_inputs(d)
    ref = O.run(d, x)["out"]
    scale = O.run(abs_terms_desc(d, 0), x)["out"]
    nv = FusedOp(d).info()["launches"][0]["nvariants"]
    for k in range(nv):
        op = FusedOp(d, variant=k)
        dev = device_tensors(d, x)
        op.run(dev)
        torch.cuda.synchronize()
        assert_normwise(to_host(dev["out"], "f32"), ref, scale, 1e-5, f"candidate {k}")


@pytest.mark.parametrize("dims,dtype", [((2, 256, 56, 56), "f16"), ((1, 40, 9, 16), "f32"), ((3, 64, 8, 8), "bf16")])
@pytest.mark.parametrize("knobs", ["FOP_TR_PIPE=1", "FOP_TR_PIPE=1,FOP_TR_U=1", "FOP_TR_PIPE=1,FOP_TR_U=1,FOP_TR_MINB=2"])
def test_transpose_software_pipelined_bitexact(monkeypatch, dims, dtype, knobs):
    """The register transpose with the next grid-stride iteration's loads issued before the
    current tiles are stored (FOP_TR_PIPE): same tiles, same arithmetic, same bits."""
    monkeypatch.setenv("FOP_TR_TMA", "0")        # the register skeleton (16-bit default: TMA tiles)
    for kv in knobs.split(","):
        k, v = kv.split("=")
        monkeypatch.setenv(k, v)
    d = W.cfg3(*dims, dtype=dtype)
    d["tensors"]["x"]["init"] = ("special", 9)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x, autotune=0)
    assert "next iteration's loads in flight" in op.source()
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("seed", list(range(12)))
def test_column_reduction_fold_random_shapes(seed):
    """Random dense odd-row column reductions on the fold path (P = W/gcd(C, W) rows per
    aligned group, 1 to 9000 groups, plus R mod P tail rows): f16/bf16/f32
    sums of x, x*x or relu(x) (normwise, R16), maxima (bit-exact), i32 wrap-around sums
    (bit-exact); every auto-tuning candidate."""
    import math
    from harness import abs_terms_desc, assert_normwise
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    rng = np.random.default_rng(1000 + seed)
    dtype = ["f16", "bf16", "f32", "i32"][seed % 4]
    Wd = 16 // (4 if dtype in ("f32", "i32") else 2)
    C = int(rng.choice([3, 5, 7, 9, 13, 37, 99, 255, 1001, 1003, 2047, 6]))
    if C % Wd == 0:
        C += 1
    P = Wd // math.gcd(C, Wd)
    R = P * [1, 2, 17, 128, 1000, 4099, 3, 9000, 64, 257, 5000, 31][seed] + seed % P   # + tail rows
    op = "max" if seed % 3 == 2 else "sum"
    expr = [("load", 0)] if op == "max" or dtype == "i32" else \
        [[("load", 0)], [("load", 0), ("mul", 0, 0)], [("load", 0), ("relu", 0)]][seed % 3]
    d = _colred(R, C, dtype, op, expr)
    if dtype == "i32":
        d["tensors"]["x"]["init"] = ("randint", -2 ** 30, 2 ** 30, 500 + seed)
        d["tensors"]["out"]["dtype"] = "i32"
    x = W.make_inputs(d)
    ref = O.run(d, x)["out"]
    assert "fold_flag" in FusedOp(d).source(), (R, C, dtype)
    nv = FusedOp(d).info()["launches"][0]["nvariants"]
    for k in range(nv):
        got, o = run_gpu(d, x, variant=k)
        tag = f"R={R} C={C} {dtype} {op} candidate {k}"
        if op == "max" or dtype == "i32":
            assert_bitexact(got["out"], ref, tag)
        else:
            assert_normwise(got["out"], ref, O.run(abs_terms_desc(d, 0), x)["out"], 1e-5, tag)
