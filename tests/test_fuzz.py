"""Randomised operators (tests/fuzz_gen.py) through the whole path.

CPU: every random operator validates, plans and compiles for sm_100a (NVRTC).
GPU: every random operator matches the oracle — ASSIGN outputs bit for bit
(IEEE-exact ops, divisions included: the 16-bit fast form for a
loop-invariant divisor is Markstein's correction, equal to IEEE division,
DESIGN §4; integer statements, reading R30), max reductions bit for bit,
sums normwise (R16).
"""
import numpy as np
import pytest

import workloads as W
from oracle import oracle as O

from fuzz_gen import random_op

N_CPU, N_GPU = 80, 160


def _ops(n, seed):
    rng = np.random.default_rng(seed)
    return [random_op(rng) for _ in range(n)]


def test_random_ops_plan_and_compile():
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    classes = set()
    for d in _ops(N_CPU, 2026):
        op = FusedOp(d, autotune=0)
        for li in op.info()["launches"]:
            classes.add(li["class"])
            assert li["grid"] >= 1 and li["block"] >= 32
    assert classes >= {"ew", "row_reduce", "col_reduce"}


@pytest.mark.gpu
def test_random_ops_match_oracle():
    from harness import run_gpu, assert_bitexact, assert_ulp, assert_normwise, abs_terms_desc
    for i, d in enumerate(_ops(N_GPU, 4242)):
        x = W.make_inputs(d)
        got, op = run_gpu(d, x)
        ref = O.run(d, x, outputs=W.alloc_outputs(d))
        for si, st in enumerate(d["stmts"]):
            n = st["write"][0]
            t = d["tensors"][n]
            if t["role"] != "out":
                continue
            tag = f"case {i} ({d['name']}) {n}"
            # reads a statistic produced by a sum reduction: inherits its error
            from_sum = any(q["kind"] == "reduce" and q.get("op", "sum") == "sum" and
                           any(r[0] == q["write"][0] for r in st["reads"]) for q in d["stmts"][:si])
            if st["kind"] == "reduce" and st.get("op", "sum") == "sum" and t["dtype"] != "i32":   # (i32: exact)
                scale = O.run(abs_terms_desc(d, si), x)[n]
                assert_normwise(got[n], ref[n], scale, 1e-5, tag)
            elif from_sum and t["dtype"] == "f32":
                g, r = got[n].astype(np.float64), ref[n].astype(np.float64)
                assert np.all((np.abs(g - r) <= 1e-5 * np.abs(r) + 1e-30) | (np.isnan(g) & np.isnan(r))), tag
            elif t["dtype"] != "f32" and from_sum:   # (÷ is IEEE-exact in every form, fast 16-bit ones included)
                assert_ulp(got[n], ref[n], 1, tag)
            else:
                assert_bitexact(got[n], ref[n], tag)


def _table_tail_case():
    """Found by the fuzz campaign: a per-l0 shared-memory table (x1[l0] / x1[l0]
    is costly and invariant along l1) read by unroll slots past the end of the
    work — their index left the table (illegal address)."""
    return {"name": "table_tail", "loops": {"l0": 100, "l1": 7},
            "tensors": {"x0": {"shape": [7], "dtype": "f32", "role": "in", "init": ("normal", 0.0, 1.0, 1)},
                        "x1": {"shape": [100], "dtype": "f16", "role": "in", "init": ("normal", 0.0, 1.0, 2)},
                        "x2": {"shape": [7], "dtype": "f32", "role": "in", "init": ("normal", 0.0, 1.0, 3)},
                        "out": {"shape": [100, 7], "dtype": "f16", "role": "out", "strides": [8, 1]}},
            "stmts": [{"kind": "assign", "loops": ["l0", "l1"], "write": ("out", ["l0", "l1"]),
                       "reads": [("x0", ["l1"]), ("x1", ["l0"]), ("x2", ["l1"])],
                       "expr": [("load", 0), ("load", 1), ("load", 2), ("div", 1, 1), ("add", 3, 0),
                                ("add", 4, 2), ("cast", 5, "bf16")]}]}


def _long_outer_reduction_case():
    """Found by the fuzz campaign: a row reduction over two loops whose outer
    one has > 64 iterations was rejected (now a runtime loop)."""
    return {"name": "outer_red", "loops": {"a": 6, "b": 100, "c": 40},
            "tensors": {"x": {"shape": [6, 100, 40], "dtype": "f16", "role": "in", "init": ("normal", 0.0, 1.0, 4)},
                        "s": {"shape": [6], "dtype": "f32", "role": "out"}},
            "stmts": [{"kind": "reduce", "op": "sum", "loops": ["a", "b", "c"], "write": ("s", ["a"]),
                       "reads": [("x", ["a", "b", "c"])], "expr": [("load", 0)]}]}


def _long_lane_chain_case():
    """Found by the fuzz campaign (seed 5, case 119): a row reduction whose
    vector loop holds ONE vector (l3, extent 2) under 3200 outer reduction
    iterations (l0 x l2, l2 used by no access): one lane summed 6400 terms in
    sequence and exceeded the 1e-5 normwise bound (ratio 1.61).  Such lanes
    now accumulate with compensated (Kahan) summation."""
    return {"name": "long_lane_chain", "loops": {"l0": 32, "l1": 13, "l2": 100, "l3": 2},
            "tensors": {"x0": {"shape": [32, 13, 2], "dtype": "bf16", "role": "in",
                               "init": ("normal", 0.0, 1.0, 55826), "strides": [60, 4, 1]},
                        "x1": {"shape": [13, 2], "dtype": "f16", "role": "in", "init": ("normal", 0.0, 1.0, 55827)},
                        "out": {"shape": [13], "dtype": "f32", "role": "out"}},
            "stmts": [{"kind": "reduce", "op": "sum", "loops": ["l0", "l1", "l2", "l3"], "write": ("out", ["l1"]),
                       "reads": [("x0", ["l0", "l1", "l3"]), ("x1", ["l1", "l3"])],
                       "expr": [("load", 0), ("load", 1), ("const", 2.0), ("abs", 0), ("add", 3, 1)]}]}


def test_long_lane_chain_splits_lanes_or_compensates(monkeypatch):
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    # default: the lanes split the 3200 outer iterations (short chains per lane)
    src = FusedOp(_long_lane_chain_case(), autotune=0).source(0)
    assert "ro_ = sub_;" in src
    # lanes over the single vector only: one long chain, summed with compensation
    monkeypatch.setenv("FOP_ROW_SPLIT", "0")
    monkeypatch.setenv("FOP_ROW_Q", "1")
    src = FusedOp(_long_lane_chain_case(), autotune=0).source(0)
    assert "cp = fop::sub2(fop::sub2(t_" in src and "sub_" not in src.replace("__fsub_rn", "")
    assert "cp = fop::sub2" not in FusedOp(W.cfg4a(2, 8, 768), autotune=0).source(0)


@pytest.mark.gpu
def test_fuzz_regressions():
    from harness import run_gpu, assert_ulp, assert_normwise, abs_terms_desc
    d = _table_tail_case()
    x = W.make_inputs(d)
    got, _ = run_gpu(d, x)
    assert_ulp(got["out"], O.run(d, x, outputs=W.alloc_outputs(d))["out"], 1, "out")
    d = _long_outer_reduction_case()
    x = W.make_inputs(d)
    got, op = run_gpu(d, x)
    assert op.info()["launches"][0]["class"] == "row_reduce"
    assert_normwise(got["s"], O.run(d, x)["s"], O.run(abs_terms_desc(d, 0), x)["s"], 1e-5, "s")
    d = _long_lane_chain_case()
    x = W.make_inputs(d)
    for knobs in ({}, {"FOP_ROW_SPLIT": "0", "FOP_ROW_Q": "1"}):   # split lanes / one compensated chain
        import os
        old = {k: os.environ.get(k) for k in knobs}
        os.environ.update(knobs)
        try:
            got, _ = run_gpu(d, x)
        finally:
            for k, v in old.items():
                if v is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = v
        assert_normwise(got["out"], O.run(d, x)["out"], O.run(abs_terms_desc(d, 0), x)["out"], 1e-5, "out")


def _regression_descs():
    import glob
    import json
    import os
    here = os.path.join(os.path.dirname(os.path.abspath(__file__)), "fuzz_regressions")
    return [(os.path.basename(p), json.load(open(p))) for p in sorted(glob.glob(os.path.join(here, "*.json")))]


@pytest.mark.parametrize("name,d", _regression_descs())
def test_fuzz_regression_descriptors_compile(name, d):
    """Operators a fuzz campaign broke (JSON under tests/fuzz_regressions/): they plan and compile
    for sm_100a.  period_scalar_*: an EW statement flattened over an odd innermost extent that also
    reads a tensor constant along both flattened loops (round 2, seeds 35 and 37: the scalar was
    emitted as a per-element array)."""
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    FusedOp(d)


@pytest.mark.gpu
@pytest.mark.parametrize("name,d", _regression_descs())
def test_fuzz_regression_descriptors_match_oracle(name, d):
    import sys
    import os
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
    from fuzz_campaign import check
    check(d, repeat=True)


@pytest.mark.gpu
@pytest.mark.parametrize("name,d", _regression_descs())
def test_fuzz_regression_descriptors_run(name, d):
    """Every fuzz regression through the campaign's own sequence: a first (tuning) run, then
    aligned, misaligned (narrow variant) and aligned runs of the same plan, all against the
    oracle.  tma_seed41_case273: a 128x128 bf16 transpose on the TMA tiles (round 2's
    default) failed cuTensorMapEncodeTiled on one of the repeat runs."""
    import importlib.util
    import os
    spec = importlib.util.spec_from_file_location(
        "fuzz_campaign", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools",
                                      "fuzz_campaign.py"))
    fc = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(fc)
    fc.check(d, repeat=True)


def test_packed_products_are_never_contracted_into_later_adds(tmp_path):
    """fuzz seed 51 case 289: out = bf16(max(p, p) + y) with p = (x0 - x1) * x1 came out one
    bf16 ulp off because ptxas saw through max(p, p) and fused the packed product into the add
    (FFMA2).  Every packed product is now hidden at its source: the kernel's SASS has FMUL2 and
    no FFMA2 (compiled here with nvcc -fmad=false, as NVRTC compiles it)."""
    import json
    import os
    import shutil
    import subprocess
    nvcc = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    cuobjdump = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not (os.path.exists(nvcc) and os.path.exists(cuobjdump)):
        pytest.skip("needs nvcc + cuobjdump")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    d = json.load(open(os.path.join(root, "tests", "fuzz_regressions", "contract_seed51_case289.json")))
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    src = FusedOp(d, jit=0, autotune=0).source(0)
    (tmp_path / "k.cu").write_text(src)
    subprocess.run([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-fmad=false", "-cubin",
                    "-I", os.path.join(root, "paper_conf_cgo_bastoulzrlsjfjc22_b200", "csrc", "device"),
                    "-o", str(tmp_path / "k.cubin"), str(tmp_path / "k.cu")], check=True)
    sass = subprocess.run([cuobjdump, "-sass", str(tmp_path / "k.cubin")], check=True, capture_output=True,
                          text=True).stdout
    assert "FMUL2" in sass and "FFMA2" not in sass


def test_generated_kernels_have_no_zero_trip_copy_loops():
    """Lint over random operators' generated sources: no `for (i = 0; i < 0; ...)` loop — the
    shape of fuzz seed 51's bug, where a shared-memory read-out sized in 16 B chunks copied
    nothing for a thread holding 8 B and the kernel stored uninitialised registers."""
    import re
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
    pat = re.compile(r"for \((?:int|unsigned) (\w+) = 0; \1 < 0u?; ")
    bad = []
    for i, d in enumerate(_ops(300, 777)):
        op = FusedOp(d, jit=0, autotune=0)
        for k in range(len(op.info()["launches"])):
            m = pat.search(op.source(k))
            if m:
                bad.append((i, k, op.source(k)[m.start():m.start() + 120]))
    import json
    d = json.load(open(__import__("os").path.join(__import__("os").path.dirname(__file__), "fuzz_regressions",
                                                    "trsmem_seed51_case56.json")))
    assert not pat.search(FusedOp(d, jit=0, autotune=0).source(0))
    assert not bad, bad[:3]
