"""GPU parity: the CUDA path (through the C ABI) vs the oracle, element by
element, on the same seeded inputs (BASELINE.json north_star tolerances):
  * bit-exact: transposes, copies, integer moves, fp32 elementwise (same op
    order, no contraction) and every output that is a deterministic function
    of IEEE-correct ops (cfg2's BN: / sqrt * + relu, RNE cast);
  * <= 1 fp16/bf16 ulp where a transcendental (GELU) precedes the cast;
  * reductions: normwise |gpu - ref| <= tol * fin(sum |term|) (reading R16).
Sizes span several tiles plus ragged tails; full-size runs sample batch
slices (the operators are independent along the batch loop).
"""
import copy

import numpy as np
import pytest
import torch

import workloads as W
from oracle import oracle as O

from harness import (abs_terms_desc, assert_bitexact, assert_normwise, assert_ulp, run_gpu,
                     device_tensors, to_host)

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)


def _outs(desc):
    return [n for n, t in desc["tensors"].items() if t["role"] in ("out", "inout")]


# ---------------------------------------------------------------- EW
@pytest.mark.parametrize("shape", [(4, 8, 16), (3, 5, 7), (2, 3, 1000003 // 6), (1, 1, 1), (64, 33, 40)])
def test_cfg1_ew_bitexact(shape):
    d = W.cfg1(*shape)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    ref = O.run(d, x)
    assert_bitexact(got["out"], ref["out"], "out")


def test_cfg1_bias_b_and_novec_and_orders():
    d = W.cfg1_bias_b(4, 8, 16)
    x = W.make_inputs(d)
    ref = O.run(d, x)
    for opts in [{}, {"force_width": 1}, {"coalesce_order": "memory"}, {"max_vec_bytes": 32}]:
        got, op = run_gpu(d, x, **opts)
        assert_bitexact(got["out"], ref["out"], f"out {opts}")


def test_cfg1_misaligned_pointers_use_narrow_variant():
    d = W.cfg1(4, 8, 16)
    x = W.make_inputs(d)
    ref = O.run(d, x)
    got, op = run_gpu(d, x, offset=1)      # base pointers 4 B off a 16 B boundary
    assert_bitexact(got["out"], ref["out"], "out")


@pytest.mark.parametrize("dims", [(2, 64, 112, 112), (1, 3, 7, 13), (3, 5, 4, 24)])
def test_cfg2_bn_relu_cast_bitexact(dims):
    d = W.cfg2(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    ref = O.run(d, x)
    assert_bitexact(got["y"], ref["y"], "y")


@pytest.mark.parametrize("dims", [(2, 7, 9, 64), (1, 5, 5, 96), (3, 4, 4, 8)])
def test_cfg2_nhwc_channel_tables_bitexact(dims):
    """BN on NHWC: scale/shift vary along the vector loop (c), tabulated per CTA
    in shared memory and read per element; identical IEEE ops, same bits."""
    d = W.cfg2_nhwc(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert "__shared__ __align__(16) float tbl" in op.source()
    assert_bitexact(got["y"], O.run(d, x)["y"], "y")


def test_cfg2_orders_widths_agree():
    d = W.cfg2(2, 64, 28, 28)
    x = W.make_inputs(d)
    ref = O.run(d, x)
    for opts in [{"coalesce_order": "memory"}, {"force_width": 2}, {"max_vec_bytes": 32}]:
        got, op = run_gpu(d, x, **opts)
        assert_bitexact(got["y"], ref["y"], f"y {opts}")


def test_bf16_and_casts():
    d = W.cfg1(4, 8, 64)
    d["tensors"]["out"]["dtype"] = "bf16"
    d["stmts"][0]["expr"] = d["stmts"][0]["expr"] + [("cast", 5, "f16"), ("sigmoid", 6),
                                                     ("add", 7, 5)]
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    ref = O.run(d, x)
    from harness import ordered16
    diff = np.abs(ordered16(got["out"]) - ordered16(ref["out"]))   # bf16 has fp16's sign/magnitude order
    assert diff.max() <= 1, diff.max()


# ---------------------------------------------------------------- Fig. 2 running example (N2)
@pytest.mark.parametrize("N,order", [(64, ("i", "j", "k")), (64, ("i", "k", "j")), (37, ("i", "j", "k")),
                                     (256, ("i", "j", "k"))])
def test_fig2_running_example_bitexact(N, order):
    """Y: C[i][j] = C[i][j] + B[i][k] * D[k][i][j] over k in order, X: B = A + 1
    inlined — the sequential k order is preserved, so even real-valued data
    gives the oracle's exact bits."""
    d = W.fig2_running_example(N, order_y=order)
    d["tensors"]["D"]["init"] = ("normal", 0.0, 1.0, 23)
    d["tensors"]["C"]["init"] = ("normal", 0.0, 1.0, 22)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.info()["launches"][0]["vec_loop"] == "j"
    assert_bitexact(got["C"], O.run(d, x)["C"], "C")


def test_fig2_fp16_target_rounds_every_step():
    d = W.fig2_running_example(48)
    d["tensors"]["C"]["dtype"] = "f16"
    d["tensors"]["D"]["init"] = ("normal", 0.0, 1.0, 23)
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    assert_bitexact(got["C"], O.run(d, x)["C"], "C")


# ---------------------------------------------------------------- TRANSPOSE
@pytest.mark.parametrize("dims", [(2, 256, 56, 56), (1, 24, 5, 7), (2, 40, 3, 16), (1, 8, 1, 8)])
@pytest.mark.parametrize("tma", ["0", "1"])
def test_cfg3_transpose_bitexact(monkeypatch, dims, tma):
    monkeypatch.setenv("FOP_TR_TMA", tma)       # register tiles / TMA tiles (the 16-bit default)
    d = W.cfg3(*dims)
    d["tensors"]["x"]["init"] = ("special", 9)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    ref = O.run(d, x)
    assert_bitexact(got["out"], ref["out"], "out")


@pytest.mark.parametrize("dims,move", [((2, 256, 56, 56), False), ((1, 40, 9, 13), False), ((2, 128, 8, 64), True),
                                       ((1, 64, 64, 64), False)])
def test_cfg3_tma_transpose_bitexact(monkeypatch, dims, move):
    """TMA path (cp.async.bulk.tensor, 128B swizzle, mbarrier pipeline; the 16-bit default):
    64x64 tiles with out-of-bounds edges (C=40, HW=117) must give the same bits."""
    monkeypatch.setenv("FOP_TR_TMA", "1")
    d = W.cfg3(*dims)
    d["tensors"]["x"]["init"] = ("special", 9)
    if move:
        d["stmts"][0]["expr"] = [("load", 0)]
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    li = op.info()["launches"][0]
    tma = min(dims[1], dims[2] * dims[3]) >= 64
    assert (li["block"] == 128) == tma
    ref = O.run(d, x)
    if move:
        assert np.array_equal(got["out"].view(np.uint16), ref["out"].view(np.uint16))
    else:
        assert_bitexact(got["out"], ref["out"], "out")


@pytest.mark.parametrize("tma", ["0", "1"])
def test_transpose_padded_input_rows(monkeypatch, tma):
    """NCHW input with padded rows (w stride 72 > 64): h and w no longer collapse
    (4-D tensor map on the TMA path, 3 kernel loops on the register path)."""
    monkeypatch.setenv("FOP_TR_TMA", tma)
    d = W.cfg3(2, 64, 64, 64)
    d["tensors"]["x"]["strides"] = [64 * 64 * 72, 64 * 72, 72, 1]
    d["tensors"]["x"]["init"] = ("special", 5)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


def test_cfg3_classifies_as_transpose_with_both_sides_vectorised():
    d = W.cfg3(2, 256, 56, 56)
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    info = FusedOp(d).info()["launches"][0]
    assert info["class"] == "transpose" and info["vec_loop"] == "c" and info["read_loop"] == "w"
    assert info["width"] == 8 and info["read_width"] == 8


def test_pure_move_transposes_keep_nan_payloads():
    d = W.cfg3(2, 64, 8, 8)
    d["stmts"][0]["expr"] = [("load", 0)]
    d["tensors"]["x"]["init"] = ("special", 3)
    x = W.make_inputs(d)
    x["x"].view(np.uint16)[::97] = 0x7D01           # signalling-style NaN payload
    got, _ = run_gpu(d, x)
    ref = O.run(d, x)
    assert np.array_equal(got["out"].view(np.uint16), ref["out"].view(np.uint16))


@pytest.mark.parametrize("dtype", ["f32", "i32", "bf16"])
def test_transpose2d_dtypes(dtype):
    d = W.transpose2d(64, 96, dtype)
    if dtype == "i32":
        d["tensors"]["inp"]["init"] = ("randint", -1000000, 1000000, 5)
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    ref = O.run(d, x)
    assert np.array_equal(got["out"].view(np.uint8), ref["out"].view(np.uint8))


def test_transpose_roundtrip_on_gpu():
    N, C, H, Wd = 2, 32, 6, 10
    d = W.cfg3(N, C, H, Wd, s=1.0)
    d["tensors"]["x"]["init"] = ("special", 4)
    x = W.make_inputs(d)
    t, _ = run_gpu(d, x)
    d2 = W.cfg3(N, C, H, Wd, s=1.0)
    d2["tensors"]["x"]["shape"] = [N, H, Wd, C]
    d2["tensors"]["out"]["shape"] = [N, C, H, Wd]
    d2["stmts"][0]["write"] = ("out", ["n", "c", "h", "w"])
    d2["stmts"][0]["reads"] = [("x", ["n", "h", "w", "c"])]
    back, _ = run_gpu(d2, {"x": t["out"]})
    assert_bitexact(back["out"], x["x"], "roundtrip")


@pytest.mark.parametrize("dims,cls", [((2, 56, 56, 256), "transpose"), ((3, 7, 9, 64), "transpose"),
                                      ((1, 14, 14, 40), "transpose"), ((2, 5, 8, 24), "transpose"),
                                      ((2, 7, 7, 2048), "transpose")])
@pytest.mark.parametrize("tma", ["0", "1"])
def test_nhwc_to_nchw_bitexact(monkeypatch, dims, cls, tma):
    """The reverse layout change: d_v absorbs h after w (one contiguous run of
    H*W on both sides), so the store tiles span whole NCHW planes.  An odd
    H*W (63, 49) cannot carry store vectors: flat output tiles through shared
    memory."""
    monkeypatch.setenv("FOP_TR_TMA", tma)
    d = W.nhwc_to_nchw(*dims, s=0.5)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.info()["launches"][0]["class"] == cls
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("dims,dtype", [((2, 2048, 7, 7), "f16"), ((3, 64, 3, 3), "f16"), ((2, 40, 5, 7), "f32"),
                                        ((3, 24, 7, 7), "bf16"), ((2, 1024, 1, 7), "f16")])
def test_transpose_odd_planes_via_shared_memory(dims, dtype):
    """NCHW -> NHWC with an odd H*W (a 7x7 plane: 98 B rows cannot carry
    vectors): flat tiles through shared memory, bit-exact."""
    d = W.cfg3(*dims, dtype=dtype)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.selected(0)[0].startswith("fop_transpose_smem")
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("dims,dtype", [((2, 3, 16, 24), "f16"), ((2, 3, 8, 8), "f32"), ((2, 5, 8, 16), "bf16"),
                                        ((1, 3, 224, 224), "f16")])
def test_transpose_tiny_channels_via_shared_memory(dims, dtype):
    """NCHW -> NHWC of an input layer (C = 3): no store vector along c, so the
    output tile (whole NHWC rows of 3 channels) is written flat from shared
    memory; bit-exact."""
    d = W.cfg3(*dims, dtype=dtype)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.selected(0)[0].startswith("fop_transpose_smem")
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("mirror", [False, True])
def test_transpose_smem_pure_move_keeps_nan_payloads_both_ways(mirror):
    d = W.nhwc_to_nchw(2, 7, 7, 64, s=1.0) if mirror else W.cfg3(2, 64, 7, 7, s=1.0)
    d["stmts"][0]["expr"] = [("load", 0)]
    d["tensors"]["x"]["init"] = ("special", 4)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.selected(0)[0].startswith("fop_transpose_smem")
    assert np.array_equal(got["out"].view(np.uint16), O.run(d, x)["out"].view(np.uint16))


def test_transpose_smem_pure_move_keeps_nan_payloads():
    d = W.cfg3(2, 64, 7, 7, s=1.0)
    d["stmts"][0]["expr"] = [("load", 0)]
    d["tensors"]["x"]["init"] = ("special", 4)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.selected(0)[0].startswith("fop_transpose_smem")
    assert np.array_equal(got["out"].view(np.uint16), O.run(d, x)["out"].view(np.uint16))


# ---------------------------------------------------------------- ROW_REDUCE
def _check_rowstats(d, x, got):
    ref = O.run(d, x)
    assert_ulp(got["y"], ref["y"], 1, "y")
    # statistics of the GPU's own y, recomputed by the oracle: isolates the
    # reduction from the GELU's last-bit rounding
    d2 = copy.deepcopy(d)
    d2["tensors"]["y"]["role"] = "in"
    xin = dict(x)
    xin["y"] = got["y"]
    ref2 = O.run(d2, xin, stmts=[1, 2])
    for si, name in [(1, "mean"), (2, "var")]:
        scale = O.run(abs_terms_desc(d2, si), xin, stmts=[1, 2])[name]
        assert_normwise(got[name], ref2[name], scale, 1e-5, name)
        assert_normwise(got[name], ref[name], O.run(abs_terms_desc(d, si), x)[name], 2e-3, name)


@pytest.mark.parametrize("dims", [(2, 64, 768), (1, 7, 200), (3, 5, 100), (1, 3, 24), (1, 2, 4096)])
def test_cfg4a_bias_gelu_rowstats(dims):
    d = W.cfg4a(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.info()["launches"][0]["class"] == "row_reduce"
    _check_rowstats(d, x, got)


@pytest.mark.parametrize("knobs", [(160, 5), (800, 1), (96, 8)])
def test_cfg4a_row_block_geometries(monkeypatch, knobs):
    """ROW_REDUCE with warp counts per block that are not powers of two (the
    auto-tuner's balanced-rounds candidate: 5 x 160 threads per SM)."""
    monkeypatch.setenv("FOP_BLOCK", str(knobs[0]))
    monkeypatch.setenv("FOP_ROW_MINB", str(knobs[1]))
    d = W.cfg4a(3, 129, 768)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x, autotune=0)
    assert op.info()["launches"][0]["block"] == knobs[0]
    _check_rowstats(d, x, got)


def _rowsum(R, C, dtype="f16", op="sum"):
    return {
        "name": "rowsum", "loops": {"r": R, "c": C},
        "tensors": {"x": {"shape": [R, C], "dtype": dtype, "role": "in", "init": ("normal", 0.0, 1.0, 5),
                          "strides": None},
                    "out": {"shape": [R], "dtype": "f32", "role": "out", "init": None, "strides": None}},
        "stmts": [{"kind": "reduce", "op": op, "loops": ["r", "c"], "write": ("out", ["r"]),
                   "reads": [("x", ["r", "c"])], "expr": [("load", 0)]}],
    }


@pytest.mark.parametrize("R,C,dtype,op,P", [(1000, 64, "f16", "sum", 4), (4099, 16, "f32", "sum", 8),
                                            (777, 24, "f16", "max", 8), (50, 8, "bf16", "sum", 32),
                                            (33, 64, "f32", "sum", 2)])
def test_short_rows_share_a_warp(R, C, dtype, op, P):
    """Rows of fewer than 16 vectors: P rows per warp, 32/P lanes each, group
    butterflies; ragged row counts leave part of the last warp without a row."""
    d = _rowsum(R, C, dtype, op)
    x = W.make_inputs(d)
    got, o = run_gpu(d, x)
    assert f"{P} rows per warp" in o.source()
    ref = O.run(d, x)["out"]
    if op == "max":
        assert np.array_equal(got["out"], ref)
    else:
        assert_normwise(got["out"], ref, O.run(abs_terms_desc(d, 0), x)["out"], 1e-5 if dtype == "f32" else 2e-3, "out")


def test_short_row_layernorm_statistics():
    """cfg4a's bias + GELU + mean/var with 64-wide rows (4 rows per warp)."""
    d = W.cfg4a(3, 100, 64)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert "4 rows per warp" in op.source()
    _check_rowstats(d, x, got)


@pytest.mark.parametrize("dims", [(2, 64, 771), (1, 9, 1023), (3, 5, 45)])
def test_cfg4a_odd_rows_peeled(dims):
    """Rows of odd length: each row shifted to its first 16-byte-aligned
    element, 8-vectors in between, head and tail elements scalar."""
    d = W.cfg4a(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert "pe_s" in op.source()
    _check_rowstats(d, x, got)


@pytest.mark.parametrize("name,kw", [("vocab_softmax", {"R": 5, "V": 50257}), ("bert_layernorm", {"B": 1, "S": 37, "H": 1023}),
                                     ("vocab_softmax", {"R": 3, "V": 30522})])
def test_odd_row_softmax_layernorm_peeled(name, kw):
    from test_n4_ops import _assert_layernorm
    d = W.N4[name](**kw)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert "pe_s" in op.source()
    ref = O.run(d, x)
    for n, v in got.items():
        if name == "bert_layernorm":
            _assert_layernorm(d, x, v, ref[n])
        else:
            assert_ulp(v, ref[n], 1, n)


def test_peeled_rows_shift_follows_the_row_variant_access():
    """Fuzz seed 17 case 231: a row-invariant vector (bf16 x0[l1]) listed
    before the padded rows (f16 x1, pitch 102): the per-row shift must come
    from x1, not from x0 (misaligned vector loads otherwise)."""
    d = {"name": "peel_ref", "loops": {"l0": 100, "l1": 100},
         "tensors": {"x0": {"shape": [100], "dtype": "bf16", "role": "in", "init": ("normal", 0.0, 1.0, 1), "strides": [1]},
                     "x1": {"shape": [100, 100], "dtype": "f16", "role": "in", "init": ("normal", 0.0, 1.0, 2),
                            "strides": [102, 1]},
                     "out": {"shape": [100], "dtype": "f32", "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "reduce", "op": "sum", "loops": ["l0", "l1"], "write": ("out", ["l0"]),
                    "reads": [("x0", ["l1"]), ("x1", ["l0", "l1"])], "expr": [("load", 0), ("load", 1), ("mul", 0, 1)]}]}
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert "pe_s" in op.source()
    assert_normwise(got["out"], O.run(d, x)["out"], O.run(abs_terms_desc(d, 0), x)["out"], 2e-3, "out")


def test_odd_rows_misaligned_pointers_use_narrow_variant():
    d = W.cfg4a(2, 16, 771)
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x, offset=1)
    _check_rowstats(d, x, got)


def test_row_closed_forms_on_gpu():
    d = W.cfg4a(1, 4, 768)
    d["stmts"][0]["expr"] = [("load", 0)]
    d["stmts"][0]["reads"] = [("x", ["b", "s", "h"])]
    x = {"x": np.tile(np.arange(768, dtype=np.float16), 4), "bias": np.zeros(768, np.float16)}
    got, _ = run_gpu(d, x)
    assert np.all(got["mean"] == np.float32(383.5))
    assert np.allclose(got["var"], (768 ** 2 - 1) / 12, rtol=1e-6)


# ---------------------------------------------------------------- COL_REDUCE
@pytest.mark.parametrize("dims", [(4096, 1024), (1000, 40), (65536, 8), (33, 1024), (5, 3)])
def test_cfg4b_colsum(dims):
    d = W.cfg4b(*dims)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    ref = O.run(d, x)
    scale = O.run(abs_terms_desc(d, 0), x)["out"]
    assert_normwise(got["out"], ref["out"], scale, 1e-5, "out")


def test_colsum_ones_exact_and_deterministic():
    d = W.cfg4b(65536, 1024, init=("ones",))
    x = W.make_inputs(d)
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    op = FusedOp(d)
    dev = device_tensors(d, x)
    op.run(dev)
    first = dev["out"].clone()
    assert torch.all(first == 65536.0)
    d2 = W.cfg4b(65536, 1024)
    x2 = W.make_inputs(d2)
    op2 = FusedOp(d2)
    dev2 = device_tensors(d2, x2)
    runs = []
    for _ in range(3):
        op2.run(dev2)
        runs.append(dev2["out"].clone())
    torch.cuda.synchronize()
    assert all(torch.equal(runs[0], r) for r in runs[1:])   # fixed-order trees


def test_reduce_max_col_and_row():
    d = W.cfg4b(3000, 72)
    d["stmts"][0]["op"] = "max"
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    assert_bitexact(got["out"], O.run(d, x)["out"], "colmax")
    d = W.cfg4a(2, 8, 256)
    d["stmts"][1]["op"] = "max"
    d["stmts"][1]["finalize"] = []
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    ref = O.run(d, x)
    assert_ulp(got["y"], ref["y"], 1, "y")


# ---------------------------------------------------------------- full sizes (launch config of bench.py)
def _slice_batch(desc, x, got, loop, idx):
    """Oracle on batch index `idx` of `loop` vs the GPU's full-size output."""
    d1 = copy.deepcopy(desc)
    d1["loops"][loop] = 1
    xs, gs = {}, {}
    for n, t in desc["tensors"].items():
        st = W.tensor_strides(t)
        # the batch loop indexes dim 0 of every batched tensor in these configs
        if t["shape"][0] == desc["loops"][loop] and len(t["shape"]) > 1:
            d1["tensors"][n]["shape"] = [1] + t["shape"][1:]
            sl = slice(idx * st[0], (idx + 1) * st[0])
        else:
            sl = slice(None)
        if t["role"] in ("in", "inout"):
            xs[n] = x[n][sl]
        if t["role"] in ("out", "inout"):
            gs[n] = got[n][sl]
    return d1, xs, gs


@pytest.mark.parametrize("cfg,loop,out", [("cfg2", "n", "y"), ("cfg3", "n", "out")])
def test_full_size_sampled_bitexact(cfg, loop, out):
    d = W.CONFIGS[cfg]()
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    for idx in (0, d["loops"][loop] // 2 + 3, d["loops"][loop] - 1):
        d1, xs, gs = _slice_batch(d, x, got, loop, idx)
        assert_bitexact(gs[out], O.run(d1, xs)[out], f"{cfg} {loop}={idx}")


def test_full_size_cfg4a_sampled():
    d = W.cfg4a()
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    for idx in (0, 40, 63):
        d1, xs, gs = _slice_batch(d, x, got, "b", idx)
        gs["mean"] = got["mean"][idx * 512:(idx + 1) * 512]
        gs["var"] = got["var"][idx * 512:(idx + 1) * 512]
        d1["tensors"]["mean"]["shape"] = [1, 512]
        d1["tensors"]["var"]["shape"] = [1, 512]
        _check_rowstats(d1, xs, gs)


def test_full_size_cfg4b():
    d = W.cfg4b()
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    ref = O.run(d, x)
    scale = O.run(abs_terms_desc(d, 0), x)["out"]
    assert_normwise(got["out"], ref["out"], scale, 1e-5, "out")


# ---------------------------------------------------------------- end-to-end ABI path
def test_run_host_end_to_end():
    d = W.cfg2(2, 8, 16, 16)
    x = W.make_inputs(d)
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    from harness import TORCH_DT
    op = FusedOp(d)
    dev = device_tensors(d, x)
    host = {"x": torch.from_numpy(x["x"]).pin_memory()}
    for n in ("gamma", "beta", "mean", "var"):
        host[n] = torch.from_numpy(x[n]).pin_memory()
    host["y"] = torch.empty(dev["y"].numel(), dtype=TORCH_DT["f16"]).pin_memory()
    dev["x"].zero_()
    op.run_host(host, dev)
    torch.cuda.synchronize()
    assert_bitexact(host["y"].numpy(), O.run(d, x)["y"], "y")


def _host_dev(d, x):
    """Pinned host buffers (inputs from x, outputs NaN-filled) + empty device buffers."""
    outs = W.alloc_outputs(d)
    host, dev = {}, {}
    for n, t in d["tensors"].items():
        if t["role"] == "temp":
            continue
        buf = x[n] if t["role"] in ("in", "inout") else outs[n]
        host[n] = torch.from_numpy(np.ascontiguousarray(buf)).pin_memory()
        dev[n] = torch.empty_like(host[n], device="cuda")
    return host, dev


def test_run_host_many_pipelined():
    """fop_run_host_many: independent plans, copies pipelined over two internal
    streams and reordered (Johnson's rule); every result equals the oracle's,
    and a second call on fresh inputs in the same buffers sees only them."""
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, run_host_many
    descs = [W.cfg2(2, 8, 16, 16), W.cfg3(2, 16, 8, 8), W.cfg1(3, 5, 7), W.cfg4b(300, 64)]
    ops = [FusedOp(d) for d in descs]
    for seed_offset in (0, 7):
        xs = [W.make_inputs(d, seed_offset=seed_offset) for d in descs]
        hd = [_host_dev(d, x) for d, x in zip(descs, xs)]
        run_host_many([(op, h, dv) for op, (h, dv) in zip(ops, hd)])
        torch.cuda.synchronize()
        for d, x, (h, _) in zip(descs, xs, hd):
            ref = O.run(d, x)
            for n in _outs(d):
                if d["stmts"][-1]["kind"] == "reduce":
                    scale = O.run(abs_terms_desc(d, 0), x)[n]
                    assert_normwise(h[n].numpy(), ref[n], scale, 1e-5, n)
                else:
                    assert_bitexact(h[n].numpy(), ref[n], f"{d['name']} {n}")


@pytest.mark.parametrize("warm", [True, False])
def test_cuda_graph_capture_and_replay(warm):
    """fop_run inside torch.cuda.graph capture: replays follow the buffers'
    current contents.  warm=False: the plan's first run (module load, no
    auto-tuning while capturing) happens inside the capture."""
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    descs = [W.cfg2(2, 8, 16, 16), W.cfg3(2, 16, 8, 8), W.cfg4a(1, 7, 200), W.cfg4b(300, 64)]
    ops = [FusedOp(d) for d in descs]
    xs = [W.make_inputs(d) for d in descs]
    devs = [device_tensors(d, x) for d, x in zip(descs, xs)]
    wss = [op._workspace(torch.device("cuda"), torch.cuda.current_stream()) for op in ops]
    if warm:
        for op, dv, ws in zip(ops, devs, wss):
            op.run(dv, workspace=ws)
        torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for op, dv, ws in zip(ops, devs, wss):
            op.run(dv, workspace=ws)
    for seed_offset in (3, 11):
        xs = [W.make_inputs(d, seed_offset=seed_offset) for d in descs]
        for d, x, dv in zip(descs, xs, devs):
            for n, t in d["tensors"].items():
                if t["role"] in ("in", "inout"):
                    dv[n].copy_(device_tensors(d, x)[n])
        g.replay()
        torch.cuda.synchronize()
        for d, x, dv in zip(descs, xs, devs):
            ref = O.run(d, x)
            for n in _outs(d):
                got = to_host(dv[n], d["tensors"][n]["dtype"])
                if d["name"].startswith("cfg4a"):
                    if n == "y":
                        assert_ulp(got, ref[n], 1, n)
                elif d["stmts"][-1]["kind"] == "reduce":
                    scale = O.run(abs_terms_desc(d, 0), x)[n]
                    assert_normwise(got, ref[n], scale, 1e-5, n)
                else:
                    assert_bitexact(got, ref[n], f"{d['name']} {n}")


@pytest.mark.parametrize("mk", [lambda: W.cfg3(2, 64, 8, 8), lambda: W.transpose2d(128, 192, "bf16"),
                                lambda: W.nhwc_to_nchw(2, 8, 8, 64)])
@pytest.mark.parametrize("offset", [1, 4, 8])
def test_tma_transpose_misaligned_pointers_take_the_narrow_variant(mk, offset):
    """16-bit transposes plan onto TMA tiles (16 B-aligned tensor-map base addresses):
    pointers off that alignment must run the narrow variant (an EW kernel with gathers),
    never the tensor-map path; aligned runs of the same plan before and after stay exact."""
    from harness import device_tensors, to_host
    d = mk()
    x = W.make_inputs(d)
    ref = O.run(d, x)["out"]
    got, op = run_gpu(d, x, variant=0)       # the default geometry: the TMA tiles (no tuning)
    assert "TRANSPOSE via TMA" in op.source() and "tma" in op.selected(0)[0], op.selected(0)
    assert_bitexact(got["out"], ref, "aligned")
    for off in (offset, 0):
        dev = device_tensors(d, x, offset=off)
        op.run(dev)
        torch.cuda.synchronize()
        assert_bitexact(to_host(dev["out"], d["tensors"]["out"]["dtype"]), ref, f"offset {off}")


@pytest.mark.parametrize("variant", [0, -1])
@pytest.mark.parametrize("expr", [
    [("load", 0), ("const", 0.3), ("mul", 0, 1), ("const", 0.125), ("add", 2, 3)],          # x*s + t
    [("load", 0), ("load", 0), ("mul", 0, 1), ("load", 0), ("sub", 2, 3)],                  # x*x - x
    [("load", 0), ("const", -1.7), ("mul", 0, 1), ("neg", 2), ("load", 0), ("add", 3, 4)]])  # -(x*s) + x
def test_tma_transpose_products_feeding_adds_bitexact(variant, expr):
    """Products feeding adds inside the TMA transpose (launched with dynamic shared memory):
    every packed product is hidden from ptxas's contraction by OR-ing an opaque zero, which
    must be a true zero there too (FopArgs::zero; %dynamic_smem_size was not).  Bit-exact vs
    the oracle, the default TMA geometry (variant 0) and the tuner's pick."""
    d = W.cfg3(2, 128, 16, 16)
    d["stmts"][0]["expr"] = expr
    x = W.make_inputs(d)
    got, op = run_gpu(d, x, **({"variant": 0} if variant == 0 else {}))
    if variant == 0:
        assert "TRANSPOSE via TMA" in op.source()
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")
