"""Row N3: dependences, the influence-tree fallback and recurrence kernels.

CPU (not gpu): the oracle on recurrences against closed forms and library
routines; the C++ dependence analysis and the planner's schedules against the
brute-force definitions in oracle/planner_oracle.py (a schedule is
valid when every pair of iterations touching the same element keeps its
order).  GPU: the CUDA path bit-exact against the oracle.
"""

import numpy as np
import pytest

import workloads as W
from oracle import oracle as O
from oracle import planner_oracle as PO
from harness import run_gpu, assert_bitexact


def fop():
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, FopError
    return FusedOp, FopError


SMALL = {
    "scan_time": lambda: W.N3["scan_time"](B=2, T=9, H=12),
    "scan_contiguous": lambda: W.N3["scan_contiguous"](R=5, C=9),
    "shift_back": lambda: W.N3["shift_back"](N=7, C=8),
    "fibonacci": lambda: W.N3["fibonacci"](T=8, C=4),
    "ema_1d": lambda: W.N3["ema_1d"](T=12),
    "wavefront": lambda: W.N3["wavefront"](A=5, B=4, C=6),
    "skew": lambda: W.N3["skew"](A=5, B=4),
    "fig2": lambda: W.fig2_running_example(5),
}


# ------------------------------------------------------------ oracle pins
def test_oracle_scan_is_sequential_cumsum():
    """Y[b][t+1][h] = Y[b][t][h] + X[b][t+1][h] with Y = X initially is numpy's
    sequential float32 add.accumulate along t, bit for bit."""
    d = W.N3["scan_time"](B=3, T=50, H=20)
    x = W.make_inputs(d)
    got = O.run(d, x)["Y"].reshape(3, 50, 20)
    ref = np.add.accumulate(x["X"].reshape(3, 50, 20), axis=1, dtype=np.float32)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_oracle_anti_dependence_reads_old_values():
    """Y[i] = 0.5*Y[i+1] + X[i] in ascending i reads Y[i+1] before it is rewritten."""
    d = W.N3["shift_back"](N=10, C=6)
    x = W.make_inputs(d)
    got = O.run(d, x)["Y"].reshape(10, 6)
    y0, xx = x["Y"].reshape(10, 6), x["X"].reshape(10, 6)
    ref = y0.copy()
    ref[:-1] = (np.float32(0.5) * y0[1:]) + xx[:-1]
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_oracle_fibonacci_closed_form():
    d = W.N3["fibonacci"](T=30, C=3)
    x = W.make_inputs(d)
    x["Y"][:] = 0
    x["Y"].reshape(30, 3)[:2] = 1
    got = O.run(d, x)["Y"].reshape(30, 3)
    fib = [1, 1]
    while len(fib) < 30:
        fib.append(fib[-1] + fib[-2])
    assert np.array_equal(got, np.repeat(np.array(fib, np.float32)[:, None], 3, 1))


def test_oracle_ema_closed_form():
    """y[t+1] = y[t]/2 + x/2 with x = 1, y[0] = 0 gives 1 - 2^-t exactly (t <= 24)."""
    d = W.N3["ema_1d"](T=25, a=0.5)
    x = W.make_inputs(d)
    x["x"][:] = 1.0
    x["y"][:] = 0.0
    got = O.run(d, x)["y"]
    assert np.array_equal(got, np.float32(1.0) - np.float32(2.0) ** -np.arange(25, dtype=np.float32))


def test_oracle_wavefront_is_pascal_triangle():
    """Y[a+1][b+1] = Y[a][b+1] + Y[a+1][b] + X with X = 0 and unit first row
    and column is Pascal's triangle: Y[a][b] = C(a+b, a) (exact in fp32)."""
    from math import comb
    d = W.N3["wavefront"](A=9, B=8, C=3)
    x = W.make_inputs(d)
    Y = np.zeros((9, 8, 3), np.float32)
    Y[0, :], Y[:, 0] = 1.0, 1.0
    x["X"][:] = 0.0
    x["Y"] = Y.reshape(-1)
    got = O.run(d, x)["Y"].reshape(9, 8, 3)
    ref = np.array([[comb(a + b, a) for b in range(8)] for a in range(9)], np.float32)
    assert np.array_equal(got, np.repeat(ref[:, :, None], 3, 2))


# ------------------------------------------------------------ dependence analysis + schedules
def _plan(d, **kw):
    FusedOp, _ = fop()
    return FusedOp(d, jit=0, **kw)


def _dist_tuple(desc, s, dep):
    return tuple(dep["dist"].get(l, 0) for l in desc["stmts"][s]["loops"])


@pytest.mark.parametrize("name", [n for n in SMALL if n != "fig2"])
def test_recurrence_dependences_equal_bruteforce(name):
    d = SMALL[name]()
    op = _plan(d)
    s = len(d["stmts"]) - 1
    cpp = {(_dist_tuple(d, s, dep), "anti" if dep["anti"] else "flow") for dep in op.info()["stmts"][s]["deps"]}
    assert cpp == PO.distance_set(d, s)


@pytest.mark.parametrize("name", list(SMALL))
def test_planned_schedule_is_valid_by_definition(name):
    d = SMALL[name]()
    op = _plan(d)
    info = op.info()
    li = info["launches"][-1]
    s = li["main_stmt"]
    loops = d["stmts"][s]["loops"]
    par = [l for l in loops if l not in li["seq"]]
    assert li["seq"], "a statement with dependences must get sequential loops"
    assert PO.schedule_valid(d, s, li["seq"], par)
    # every scenario skipped at depth 0 would have put a dependence on the vector lanes
    scen = info["stmts"][s]["scenarios"]
    pick = li["scen_pick"]
    for k in range(pick if pick >= 0 else len(scen)):
        v = scen[k][-1]
        seq0 = [l for l in loops if l != v and l in li["seq"]]
        assert not PO.schedule_valid(d, s, seq0, [l for l in loops if l not in seq0])


def test_fig2_scenario_fully_satisfied():
    """Fig. 2(c): forall i / for k / forvec j realises scenario [i, k, j] as ranked."""
    li = _plan(W.fig2_running_example(16)).info()["launches"][0]
    assert (li["vec_loop"], li["seq"], li["coal_loop"], li["scen_pick"], li["fallback"]) == ("j", ["k"], "i", 0, 0)


def test_fallback_levels():
    # contiguous-dim scan: the best scenario vectorises c, which carries the dependence
    li = _plan(W.N3["scan_contiguous"]()).info()["launches"][0]
    assert li["scen_pick"] == 1 and li["vec_loop"] == "r" and li["seq"] == ["c"]
    # only one scenario kept: none feasible -> uninfluenced schedule, no vector type
    li = _plan(W.N3["scan_contiguous"](), max_scenarios=1).info()["launches"][0]
    assert (li["fallback"], li["vec_loop"], li["width"], li["scen_pick"]) == (2, "r", 1, -1)
    # time scan: scenario [t, b, h] wants b inside t -> looser variant keeps only h
    li = _plan(W.N3["scan_time"]()).info()["launches"][0]
    assert (li["vec_loop"], li["seq"], li["fallback"]) == ("h", ["t"], 1)
    # every loop carries a dependence -> fully sequential
    for n in ("ema_1d", "skew"):
        li = _plan(W.N3[n]()).info()["launches"][0]
        assert li["fallback"] == 3 and li["vec_loop"] is None and li["grid"] == 1


def test_wavefront_sequential_order_follows_scenario():
    """Deps (1,0) and (0,1) allow either order of a, b (permutation test);
    the scenario [b, a, c] puts a innermost."""
    li = _plan(W.N3["wavefront"]()).info()["launches"][0]
    assert li["seq"] == ["b", "a"] and li["fallback"] == 0
    d = W.N3["wavefront"](A=4, B=4, C=2)
    assert PO.schedule_valid(d, 0, ["b", "a"], ["c"]) and PO.schedule_valid(d, 0, ["a", "b"], ["c"])


def test_non_uniform_self_read_rejected():
    _, FopError = fop()
    d = {"loops": {"i": 8, "j": 8},
         "tensors": {"Y": {"shape": [8, 8], "dtype": "f32", "role": "inout"}},
         "stmts": [{"kind": "assign", "loops": ["i", "j"], "write": ("Y", ["i", "j"]),
                    "reads": [("Y", ["j", "i"])], "expr": [("load", 0), ("const", 2.0), ("mul", 0, 1)]}]}
    with pytest.raises(FopError, match="non-uniform"):
        _plan(d)


def random_recurrence(rng, dtype="f32"):
    """A statement over 2-3 loops writing T (one loop per dim, random
    permutation) at offsets in {0,1,2} and reading T at 1-2 other offsets plus
    an input X."""
    nl = int(rng.integers(2, 4))
    names = ["p", "q", "r"][:nl]
    ext = {n: int(rng.integers(2, 6)) for n in names}
    perm = list(rng.permutation(nl))
    dims = [names[i] for i in perm]                       # tensor dim r iterated by loop dims[r]
    shape = [ext[n] + 2 for n in dims]
    def acc(offs):
        return [(n, int(o)) for n, o in zip(dims, offs)]
    wo = rng.integers(0, 3, nl)
    reads = []
    for _ in range(int(rng.integers(1, 3))):
        ro = rng.integers(0, 3, nl)
        if not np.array_equal(ro, wo):
            reads.append(("T", acc(ro)))
    if not reads:
        reads.append(("T", acc((wo + 1) % 3)))
    reads.append(("X", acc(wo)))
    expr = [("load", k) for k in range(len(reads))]
    cur = 0
    for k in range(1, len(reads)):
        expr.append(("add", cur, k))
        cur = len(expr) - 1
    expr.append(("const", 0.75))
    expr.append(("mul", cur, len(expr) - 1))
    return {"name": "random_recurrence", "loops": ext,
            "tensors": {"T": {"shape": shape, "dtype": dtype, "role": "inout", "init": ("normal", 0.0, 1.0, 61)},
                        "X": {"shape": shape, "dtype": dtype, "role": "in", "init": ("normal", 0.0, 1.0, 62)}},
            "stmts": [{"kind": "assign", "loops": list(names), "write": ("T", acc(wo)), "reads": reads,
                       "expr": expr}]}


def test_random_recurrences_planned_validly():
    rng = np.random.default_rng(2024)
    n_dep = 0
    for _ in range(60):
        d = random_recurrence(rng)
        op = _plan(d)
        info = op.info()
        li = info["launches"][0]
        cpp = {(_dist_tuple(d, 0, dep), "anti" if dep["anti"] else "flow") for dep in info["stmts"][0]["deps"]}
        assert cpp == PO.distance_set(d, 0), d
        par = [l for l in d["stmts"][0]["loops"] if l not in li["seq"]]
        assert PO.schedule_valid(d, 0, li["seq"], par), (d, li)
        n_dep += bool(cpp)
    assert n_dep > 30


# ------------------------------------------------------------ GPU parity
GPU_CASES = {
    "scan_time": lambda: W.N3["scan_time"](B=8, T=100, H=200),
    "scan_time_f16": lambda: W.N3["scan_time"](B=4, T=64, H=96, dtype="f16"),
    "scan_time_bf16_tail": lambda: W.N3["scan_time"](B=3, T=20, H=37, dtype="bf16"),
    "scan_contiguous": lambda: W.N3["scan_contiguous"](R=300, C=65),
    "shift_back": lambda: W.N3["shift_back"](N=40, C=72),
    "fibonacci": lambda: W.N3["fibonacci"](T=30, C=100),
    "ema_1d": lambda: W.N3["ema_1d"](T=300),
    "wavefront": lambda: W.N3["wavefront"](A=16, B=12, C=64),
    "skew": lambda: W.N3["skew"](A=12, B=9),
}


@pytest.mark.gpu
@pytest.mark.parametrize("name", list(GPU_CASES))
def test_recurrence_bitexact(name):
    d = GPU_CASES[name]()
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    ref = O.run(d, x)
    for n, t in d["tensors"].items():
        if t["role"] in ("out", "inout"):
            assert_bitexact(got[n], ref[n], n)


@pytest.mark.gpu
def test_recurrence_max_scenarios_1_width1_bitexact():
    d = W.N3["scan_contiguous"](R=64, C=33)
    x = W.make_inputs(d)
    got, op = run_gpu(d, x, max_scenarios=1)
    assert op.info()["launches"][0]["fallback"] == 2
    assert_bitexact(got["Y"], O.run(d, x)["Y"], "Y")


@pytest.mark.gpu
def test_random_recurrences_bitexact():
    rng = np.random.default_rng(77)
    for _ in range(25):
        d = random_recurrence(rng)
        x = W.make_inputs(d)
        got, _ = run_gpu(d, x)
        assert_bitexact(got["T"], O.run(d, x)["T"], "T")


@pytest.mark.gpu
def test_scan_time_bert_size_f16():
    """Cumulative sum over the sequence of a BERT-base activation [64, 512, 768] f16."""
    d = W.N3["scan_time"](B=64, T=512, H=768, dtype="f16")
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    li = op.info()["launches"][0]
    # 49152 lanes: vectors narrowed to 4 bytes so the lanes cover the SMs
    assert li["vec_loop"] == "h" and li["width"] == 2 and li["seq"] == ["t"]
    assert_bitexact(got["Y"], O.run(d, x)["Y"], "Y")
