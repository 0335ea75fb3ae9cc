"""Integer statements (reading R30) on the GPU: int32 values, + - * max min
neg abs relu and integral constants, wrap-around modulo 2^32 — bit-exact
against the oracle (BASELINE.json north_star: "bit-exact for ... integer
ops"), through every EW path: vector loop with broadcast, narrow (misaligned)
variant, transposes, read-modify-write (Fig. 2's Y) and recurrences, and through
the row and column reduction kernels (sums modulo 2^32 are exactly associative:
every tuning candidate must give the oracle's bits).

The statement model is the paper's (statements over tensors with affine
accesses); the DAG's integer semantics are this
build's reading R30, pinned on the CPU by
tests/test_oracle_ops.py against numpy's int32 arithmetic.
"""
import numpy as np
import pytest
import torch

from oracle import oracle as O

from harness import assert_bitexact, run_gpu

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

I32 = np.int32


def _t(shape, dtype="i32", role="in"):
    return {"shape": list(shape), "dtype": dtype, "role": role, "init": None, "strides": None}


def _rand(n, seed, lo=-2 ** 31, hi=2 ** 31):
    v = np.random.default_rng(seed).integers(lo, hi, n, dtype=np.int64).astype(I32)
    v[:6] = [0, -1, 2 ** 31 - 1, -2 ** 31, 1, -2 ** 31 + 1][:min(6, n)]
    return v


@pytest.mark.parametrize("shape", [(4, 8, 16), (3, 5, 7), (2, 33, 1000), (1, 1, 1)])
@pytest.mark.parametrize("offset", [0, 1])
def test_int_elementwise_with_broadcast(shape, offset):
    A, B, C = shape
    d = {"name": "iew", "loops": {"a": A, "b": B, "c": C},
         "tensors": {"x": _t([A, B, C]), "y": _t([A, B, C]), "bias": _t([C]), "out": _t([A, B, C], role="out")},
         "stmts": [{"kind": "assign", "loops": ["a", "b", "c"], "write": ("out", ["a", "b", "c"]),
                    "reads": [("x", ["a", "b", "c"]), ("bias", ["c"]), ("y", ["a", "b", "c"])],
                    # relu(max(x + bias, -y) * 3 - y) ^ ... : every integer node, wrap-around included
                    "expr": [("load", 0), ("load", 1), ("add", 0, 1), ("load", 2), ("neg", 3), ("max", 2, 4),
                             ("const", 3.0), ("mul", 5, 6), ("sub", 7, 3), ("abs", 8), ("const", -1000.0),
                             ("min", 9, 10), ("relu", 8), ("add", 11, 12)]}]}
    n = A * B * C
    x = {"x": _rand(n, 1), "y": _rand(n, 2), "bias": _rand(C, 3)}
    got, op = run_gpu(d, x, offset=offset)
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


@pytest.mark.parametrize("op", ["add", "sub", "mul", "max", "min", "neg", "abs", "relu"])
def test_each_int_node_wraps_like_the_oracle(op):
    n = 8 * 1024
    unary = op in ("neg", "abs", "relu")
    d = {"name": "i1", "loops": {"r": 8, "i": n // 8},
         "tensors": {"a": _t([8, n // 8]), "b": _t([8, n // 8]), "out": _t([8, n // 8], role="out")},
         "stmts": [{"kind": "assign", "loops": ["r", "i"], "write": ("out", ["r", "i"]),
                    "reads": [("a", ["r", "i"]), ("b", ["r", "i"])],
                    "expr": [("load", 0), ("load", 1), (op, 0) if unary else (op, 0, 1)]}]}
    x = {"a": _rand(n, 4), "b": _rand(n, 5)}
    got, _ = run_gpu(d, x)
    ref = O.run(d, x)["out"]
    assert_bitexact(got["out"], ref, op)
    with np.errstate(over="ignore"):
        np_ref = {"add": x["a"] + x["b"], "sub": x["a"] - x["b"], "mul": x["a"] * x["b"],
                  "max": np.maximum(x["a"], x["b"]), "min": np.minimum(x["a"], x["b"]), "neg": -x["a"],
                  "abs": np.abs(x["a"]), "relu": np.maximum(x["a"], 0)}[op]
    assert np.array_equal(got["out"], np_ref)          # and numpy's int32 arithmetic, directly


@pytest.mark.parametrize("dims", [(2, 64, 7, 9), (1, 256, 56, 56), (3, 40, 5, 16)])
def test_int_transpose_with_arithmetic(dims):
    N, C, H, Wd = dims
    d = {"name": "itr", "loops": {"n": N, "c": C, "h": H, "w": Wd},
         "tensors": {"x": _t([N, C, H, Wd]), "out": _t([N, H, Wd, C], role="out")},
         "stmts": [{"kind": "assign", "loops": ["n", "c", "h", "w"], "write": ("out", ["n", "h", "w", "c"]),
                    "reads": [("x", ["n", "c", "h", "w"])],
                    "expr": [("load", 0), ("const", 65537.0), ("mul", 0, 1), ("const", 12345.0), ("add", 2, 3)]}]}
    x = {"x": _rand(N * C * H * Wd, 6)}
    got, op = run_gpu(d, x)
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")


def test_int_read_modify_write_fig2_pattern():
    """Fig. 2's Y in int32: C[i][j] += B[i][k] * D[k][i][j] over k in order (wrapping)."""
    N = 48
    d = {"name": "irmw", "loops": {"i": N, "j": N, "k": N},
         "tensors": {"B": _t([N, N]), "C": _t([N, N], role="inout"), "D": _t([N, N, N])},
         "stmts": [{"kind": "assign", "loops": ["i", "j", "k"], "write": ("C", ["i", "j"]),
                    "reads": [("C", ["i", "j"]), ("B", ["i", "k"]), ("D", ["k", "i", "j"])],
                    "expr": [("load", 0), ("load", 1), ("load", 2), ("mul", 1, 2), ("add", 0, 3)]}]}
    x = {"B": _rand(N * N, 7), "C": _rand(N * N, 8), "D": _rand(N * N * N, 9)}
    got, _ = run_gpu(d, x)
    assert_bitexact(got["C"], O.run(d, x)["C"], "C")


def test_int_recurrence_prefix_sum():
    """y[b][t] = y[b][t-1] + x[b][t] (a scan along t, row N3) in int32, wrapping."""
    Bn, T = 64, 300
    d = {"name": "iscan", "loops": {"b": Bn, "t": T - 1},
         "tensors": {"x": _t([Bn, T]), "y": _t([Bn, T], role="inout")},
         "stmts": [{"kind": "assign", "loops": ["b", "t"], "write": ("y", ["b", ("t", 1)]),
                    "reads": [("y", ["b", "t"]), ("x", ["b", ("t", 1)])],
                    "expr": [("load", 0), ("load", 1), ("add", 0, 1)]}]}
    x = {"x": _rand(Bn * T, 10, -2 ** 30, 2 ** 30), "y": _rand(Bn * T, 11)}
    got, op = run_gpu(d, x)
    assert op.info()["launches"][0]["seq"] == ["t"]
    assert_bitexact(got["y"], O.run(d, x)["y"], "y")


def _ired(R, C, op, axis, expr=None):
    return {"name": "ired", "loops": {"r": R, "c": C},
            "tensors": {"x": _t([R, C]), "out": _t([C] if axis == "col" else [R], role="out")},
            "stmts": [{"kind": "reduce", "op": op, "loops": ["r", "c"],
                       "write": ("out", ["c"] if axis == "col" else ["r"]), "reads": [("x", ["r", "c"])],
                       "expr": expr or [("load", 0), ("const", 3.0), ("mul", 0, 1)]}]}


@pytest.mark.parametrize("R,C", [(65536, 1024), (1000, 13), (7, 40000), (100000, 8), (3, 5), (4096, 1001), (4098, 1002)])
@pytest.mark.parametrize("op", ["sum", "max"])
@pytest.mark.parametrize("axis", ["col", "row"])
def test_int_reductions_bit_exact_every_candidate(R, C, op, axis):
    """i32 REDUCE (R30): sums modulo 2^32 are exactly associative, so the row and column
    kernels' butterflies, cross-warp / cluster / cross-chunk combines give the oracle's bits
    in any order — checked for every auto-tuning candidate (different association orders)."""
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    d = _ired(R, C, op, axis)
    x = {"x": _rand(R * C, 12)}
    ref = O.run(d, x)["out"]
    nv = FusedOp(d).info()["launches"][0]["nvariants"]
    for k in range(nv):
        got, op_ = run_gpu(d, x, variant=k)
        assert_bitexact(got["out"], ref, f"candidate {k} {op_.selected(0)[0]}")
    with np.errstate(over="ignore"):
        m = x["x"].reshape(R, C).astype(np.int64) * 3
        red = m.sum(0 if axis == "col" else 1) if op == "sum" else m.max(0 if axis == "col" else 1)
    if op == "max":                                   # numpy: max of the wrapped products
        red = ((x["x"].reshape(R, C) * np.int32(3)).astype(np.int32)).max(0 if axis == "col" else 1)
    red = red.astype(np.int64)
    assert np.array_equal(got["out"], ((red + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(I32))


def test_int_column_sum_misaligned_uses_the_narrow_variant():
    d = _ired(777, 1001, "sum", "col", [("load", 0)])
    x = {"x": _rand(777 * 1001, 13)}
    got, op = run_gpu(d, x, offset=1)
    assert_bitexact(got["out"], O.run(d, x)["out"], "out")
