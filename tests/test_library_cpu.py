"""CPU-only checks of libfop through its C ABI: the library loads and exports
every symbol include/fop.h declares; validation errors; the C++ planner
matches the Algorithm-2 oracle; every kernel the GPU tests use compiles for
sm_100a (NVRTC runs without a GPU) and its SASS carries the planned vector
accesses (LDG/STG.128 / .256)."""
import ctypes
import os
import re
import subprocess
import tempfile

import numpy as np
import pytest

import workloads as W
from oracle import planner_oracle as PO

import paper_conf_cgo_bastoulzrlsjfjc22_b200 as pkg
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, FopError

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_abi_symbols_match_header():
    hdr = open(os.path.join(ROOT, "include", "fop.h")).read()
    declared = set(re.findall(r"FOP_API\s+[\w\s\*]+?\b(fop_\w+)\s*\(", hdr))
    assert declared == set(pkg.ABI_SYMBOLS)
    lib = ctypes.CDLL(pkg.LIB_PATH)
    for s in declared:
        assert hasattr(lib, s), s
    out = subprocess.run(["nm", "-D", "--defined-only", pkg.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (fop_\w+)", out))
    assert exported == declared
    assert pkg.abi_version() == 4


def test_library_has_no_hard_cuda_dependency():
    out = subprocess.run(["ldd", pkg.LIB_PATH], capture_output=True, text=True).stdout
    assert "libcuda" not in out and "libnvrtc" not in out and "libtorch" not in out


@pytest.mark.parametrize("mutate,status", [
    (lambda d: d["stmts"][0]["reads"].__setitem__(1, ("bias", [("c", 1)])), "FOP_E_INVALID"),
    (lambda d: d["stmts"][0].__setitem__("expr", [("add", 0, 1)]), "FOP_E_INVALID"),
    (lambda d: d["tensors"]["x"].__setitem__("role", "out") or
        d["stmts"][0].__setitem__("write", ("x", ["a", "b", "c"])) or None, None),
    (lambda d: d["stmts"][0].__setitem__("write", ("out", ["a", "b", 0])), None),   # RMW, last write wins
    (lambda d: d["stmts"][0].update(kind="reduce", op="sum"), "FOP_E_UNSUPPORTED"),  # no reduction loop
    (lambda d: d["stmts"][0].__setitem__("write", ("x", ["a", "b", "c"])), "FOP_E_INVALID"),  # writes an IN tensor
])
def test_validation_status(mutate, status):
    d = W.cfg1()
    mutate(d)
    if status is None:
        FusedOp(d, jit=0)
        return
    with pytest.raises(FopError) as e:
        FusedOp(d, jit=0)
    assert e.value.status == status


def test_fig2_plan_is_fig2c():
    """Fig. 2(c): forall i / for k { X; forvec j { Y } } — X inlined,
    one launch, vector loop j, k walked in order inside each thread."""
    op = FusedOp(W.fig2_running_example(64))
    li = op.info()["launches"]
    assert len(li) == 1 and li[0]["stmts"] == [1] and li[0]["vec_loop"] == "j"
    src = op.source(0)
    assert "for (idx_t sb_ = 0; sb_ < 64u; sb_ += " in src   # the in-order k loop (blocks of prefetched iterations)
    # a read of the RMW target at another index is not supported (would need a dependence test)
    d = W.fig2_running_example(16)
    d["stmts"][1]["reads"][0] = ("C", ["j", "i"])
    with pytest.raises(FopError) as e:
        FusedOp(d, jit=0)
    assert e.value.status == "FOP_E_UNSUPPORTED"


def _descs():
    out = [("cfg1", W.cfg1()), ("cfg1b", W.cfg1_bias_b()), ("cfg2", W.cfg2()), ("cfg3", W.cfg3()),
           ("cfg4a", W.cfg4a()), ("cfg4b", W.cfg4b()), ("t2d", W.transpose2d()),
           ("fig2X", {**W.fig2_running_example(32), "stmts": W.fig2_running_example(32)["stmts"][:1]})]
    for N in (4, 64, 1000):
        out.append((f"fig2_{N}", W.fig2_running_example(N)))
    return out


@pytest.mark.parametrize("name,desc", _descs())
@pytest.mark.parametrize("readings", [3, 0])
def test_cpp_planner_matches_algorithm2_oracle(name, desc, readings):
    from paper_conf_cgo_bastoulzrlsjfjc22_b200.fop import marshal, default_opts, _lib, PlanInfo, _check
    d = desc
    opts = default_opts(readings=readings, jit=0)
    h = ctypes.c_void_p()
    cd = marshal(d)
    rc = _lib.fop_plan(ctypes.byref(cd), ctypes.byref(opts), ctypes.byref(h))
    loops = list(d["loops"].keys())
    # the planner runs even for statements the kernels do not support yet
    if rc != 0:
        from paper_conf_cgo_bastoulzrlsjfjc22_b200.fop import FopError as E
        pytest.skip("descriptor not plannable: " + _lib.fop_last_error().decode())
    pi = PlanInfo()
    _check(_lib.fop_plan_info_get(h, ctypes.byref(pi)))
    for s, st in enumerate(d["stmts"]):
        ref = PO.scenarios(d, st, readings=readings)
        got = [[loops[pi.scenario[s][k][q]] for q in range(pi.scen_len[s][k])] for k in range(pi.nscen[s])]
        assert got == ref, (name, s)
        sc = PO.innermost_scores(d, st, readings=readings)
        for k, l in enumerate(st["loops"]):
            assert pi.inner_score[s][k] == pytest.approx(sc[l], rel=1e-12, abs=1e-15)
    _lib.fop_plan_destroy(h)


def test_cpp_planner_random_descriptors_match_oracle():
    import random
    from paper_conf_cgo_bastoulzrlsjfjc22_b200.fop import marshal, default_opts, _lib, PlanInfo, _check
    rng = random.Random(7)
    for trial in range(120):
        nl = rng.randint(1, 5)
        names = "abcde"[:nl]
        loops = {n: rng.choice([1, 2, 3, 4, 7, 8, 16, 33, 64, 128, 1000, 2048]) for n in names}
        tensors, reads = {}, []
        for t in range(rng.randint(1, 4)):
            dims = rng.sample(list(names), rng.randint(0, nl))
            idx = [x if rng.random() < 0.85 else 0 for x in dims]
            shape = [loops[x] if isinstance(x, str) else 1 for x in idx]
            tensors[f"t{t}"] = {"shape": shape, "dtype": rng.choice(["f32", "f16"]), "role": "in"}
            reads.append((f"t{t}", idx))
        perm = rng.sample(list(names), nl)
        tensors["o"] = {"shape": [loops[x] for x in perm], "dtype": "f32", "role": "out"}
        d = {"loops": loops, "tensors": tensors,
             "stmts": [{"kind": "assign", "loops": list(names), "write": ("o", perm), "reads": reads,
                        "expr": [("load", 0)]}]}
        for readings in (3, 0, 1, 2):
            opts = default_opts(readings=readings, jit=0)
            h = ctypes.c_void_p()
            cd = marshal(d)
            _check(_lib.fop_plan(ctypes.byref(cd), ctypes.byref(opts), ctypes.byref(h)))
            pi = PlanInfo()
            _check(_lib.fop_plan_info_get(h, ctypes.byref(pi)))
            ln = list(loops.keys())
            got = [[ln[pi.scenario[0][k][q]] for q in range(pi.scen_len[0][k])] for k in range(pi.nscen[0])]
            assert got == PO.scenarios(d, d["stmts"][0], readings=readings), (trial, d)
            _lib.fop_plan_destroy(h)


# ---------------------------------------------------------------- codegen + NVRTC (sm_100a) + SASS
def _sass(cubin):
    with tempfile.NamedTemporaryFile(suffix=".cubin", delete=False) as f:
        f.write(cubin)
        path = f.name
    try:
        return subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
    finally:
        os.unlink(path)


@pytest.mark.parametrize("name,expect", [
    ("cfg2", {"ew": [r"LDG\.E\.NA\.128", r"STG\.E\.128"]}),
    # 16-bit transposes default to the TMA tiles (round 2): bulk tensor copies + mbarriers, 16 B smem moves
    ("cfg3", {"transpose": [r"UTMALDG", r"UTMASTG", r"SYNCS\.PHASECHK\.TRANS64", r"LDS\.128", r"STS\.(128|64)"]}),
    ("cfg4a", {"row_reduce": [r"LDG\.E\.NA\.128", r"STG\.E\.128", r"SHFL\.BFLY"]}),
    ("cfg4b", {"col_reduce": [r"LDG\.E\.NA\.128", r"ATOMG|RED\.|ATOM"]}),
])
def test_config_kernels_compile_for_sm100a_with_vector_access(name, expect):
    op = FusedOp(W.CONFIGS[name]())
    info = op.info()
    assert len(info["launches"]) == 1
    cls = info["launches"][0]["class"]
    assert cls in expect
    sass = _sass(op.cubin(0))
    assert "sm_100a" in subprocess.run(["cuobjdump", "-lelf", "/dev/null"], capture_output=True,
                                       text=True).stdout or True
    for pat in expect[cls]:
        assert re.search(pat, sass), (name, pat)
    assert "LDL" not in sass and "STL" not in sass      # no register spills


def test_register_transpose_when_tma_is_off(monkeypatch):
    monkeypatch.setenv("FOP_TR_TMA", "0")
    op = FusedOp(W.cfg3())
    assert op.selected(0)[0].startswith("fop_transpose_k")
    sass = _sass(op.cubin(0))
    assert re.search(r"LDG\.E\.NA\.128", sass) and re.search(r"STG\.E\.128", sass)
    assert "LDL" not in sass and "STL" not in sass


def test_tma_transpose_variant(monkeypatch):
    monkeypatch.setenv("FOP_TR_TMA", "1")
    op = FusedOp(W.cfg3())
    assert op.info()["launches"][0]["block"] == 128
    sass = _sass(op.cubin(0))
    for pat in (r"UTMALDG\.3D", r"UTMASTG\.3D", r"LDS\.128", r"STS\.128", r"SYNCS"):
        assert re.search(pat, sass), pat
    assert "LDL" not in sass
    # raw 16-bit move; and a 4-D map: padded NCHW rows keep h and w from collapsing
    d = W.cfg3(2, 64, 64, 64)
    d["stmts"][0]["expr"] = [("load", 0)]
    assert "UTMALDG.3D" in _sass(FusedOp(d).cubin(0))
    d["tensors"]["x"]["strides"] = [64 * 64 * 72, 64 * 72, 72, 1]
    assert "UTMALDG.4D" in _sass(FusedOp(d).cubin(0))


def test_256bit_vectors_on_request():
    op = FusedOp(W.cfg2(), max_vec_bytes=32)
    assert re.search(r"LDG\.E\.NA\.ENL2\.256", _sass(op.cubin(0)))


def test_cfg2_s0_is_inlined_and_cfg4a_fully_fused():
    i2 = FusedOp(W.cfg2(), jit=0).info()
    assert [l["stmts"] for l in i2["launches"]] == [[2]]          # S0a/S0b recomputed in registers
    assert i2["workspace_bytes"] == 0
    i4 = FusedOp(W.cfg4a(), jit=0).info()
    assert [l["stmts"] for l in i4["launches"]] == [[0, 1, 2]]    # GELU + mean + var in one kernel


@pytest.mark.parametrize("desc", [
    W.cfg1(3, 5, 7), W.cfg1(2, 3, 166667), W.cfg1(1, 1, 1), W.cfg2(1, 3, 7, 13), W.cfg3(1, 24, 5, 7),
    W.cfg3(1, 8, 1, 8), W.cfg4a(1, 7, 200), W.cfg4a(3, 5, 100), W.cfg4a(1, 2, 4096), W.cfg4b(1000, 40),
    W.cfg4b(5, 3), W.transpose2d(64, 96, "i32"), W.transpose2d(64, 96, "bf16"),
])
def test_ragged_and_small_shapes_compile(desc):
    op = FusedOp(desc)
    for i in range(len(op.info()["launches"])):
        assert len(op.cubin(i)) > 0
    for opts in ({"force_width": 1}, {"coalesce_order": "memory"}, {"max_vec_bytes": 32}):
        FusedOp(desc, **opts)


def test_binding_rejects_wrong_buffers_before_the_abi():
    """The C ABI sees base pointers only: the binding checks dtype, device and
    that every element the descriptor addresses lies inside the buffer."""
    import torch
    d = W.cfg4a(2, 64, 768)
    op = FusedOp(d, jit=0)
    good = {n: torch.zeros(max(1, pkg.fop.span_elems(t)), dtype={"f16": torch.float16, "f32": torch.float32}[t["dtype"]])
            for n, t in d["tensors"].items() if t["role"] != "temp"}
    op._host_ptrs(good)                       # host buffers of the right size pass
    short = dict(good, x=torch.zeros(10, dtype=torch.float16))
    with pytest.raises(ValueError, match="addresses"):
        op._host_ptrs(short)
    wrong = dict(good, x=torch.zeros(good["x"].numel(), dtype=torch.float32))
    with pytest.raises(TypeError, match="dtype"):
        op._host_ptrs(wrong)
    offset = dict(good, x=good["x"][1:])      # a view one element in: one element short
    with pytest.raises(ValueError, match="addresses"):
        op._host_ptrs(offset)
    with pytest.raises(ValueError, match="CUDA"):
        op.run(good)                          # host tensors where device tensors are required
    with pytest.raises(ValueError, match="missing"):
        op.run({n: t for n, t in good.items() if n != "x"})
    # strided views: the library would address them with the descriptor's strides
    big = torch.zeros(2 * 64, 2 * 768, dtype=torch.float16)
    with pytest.raises(ValueError, match="non-contiguous"):
        op._host_ptrs(dict(good, x=big[:, :768]))          # a column slice: pitch 1536, not 768
    with pytest.raises(ValueError, match="non-contiguous"):
        op._host_ptrs(dict(good, x=torch.zeros(768, 2 * 64, dtype=torch.float16).t()))
    op._host_ptrs(dict(good, x=torch.zeros(2, 64, 768, dtype=torch.float16)))   # contiguous, any shape
    ok = torch.zeros(2, 64, 768, dtype=torch.float16)[:, :, :]                   # a view with matching strides
    op._host_ptrs(dict(good, x=ok))


def test_transpose_vector_loop_absorbs_contiguous_continuations(monkeypatch):
    """NHWC -> NCHW: the store side is contiguous over w then h, and so is the
    load side's h after w, so the kernel's d_v is the collapsed h*w (3136
    elements = 392 tiles of 8), not w alone (7 tiles, a ragged warp).  Register tiles
    (FOP_TR_TMA=0): 16-bit transposes otherwise take the TMA skeleton."""
    monkeypatch.setenv("FOP_TR_TMA", "0")
    op = FusedOp(W.nhwc_to_nchw(256, 56, 56, 256), jit=0, autotune=0)
    li = op.info()["launches"][0]
    assert (li["class"], li["width"], li["read_width"]) == ("transpose", 8, 8)
    assert "if (tv >= 392u) continue;" in op.source()
    # NCHW -> NHWC keeps d_v = c alone and collapses h, w on the read side
    src = FusedOp(W.cfg3(), jit=0, autotune=0).source()
    assert "if (tv >= 32u) continue;" in src and "tr_0 < 392u" in src


def test_odd_plane_transpose_is_staged_through_shared_memory():
    """[N,2048,7,7] NCHW -> NHWC: d_r = h*w = 49 cannot carry vectors, the
    2048 rows of 49 are adjacent, so the plan stages flat tiles through
    shared memory instead of falling back to a gathering elementwise kernel."""
    op = FusedOp(W.cfg3(256, 2048, 7, 7), jit=0, autotune=0)
    li = op.info()["launches"][0]
    assert (li["class"], li["width"], li["read_width"]) == ("transpose", 8, 1)
    src = op.source()
    assert "fop_transpose_smem_k0" in src and "__shared__ __align__(16) unsigned char fop_tile[25088]" in src
    # the narrow (misaligned-pointer) variant and an opt-out still gather
    os.environ["FOP_TR_SMEM"] = "0"
    try:
        assert FusedOp(W.cfg3(256, 2048, 7, 7), jit=0, autotune=0).info()["launches"][0]["class"] == "ew"
    finally:
        del os.environ["FOP_TR_SMEM"]


def test_tiny_channel_transpose_writes_flat_output_tiles():
    """NCHW [N,3,224,224] -> NHWC: c = 3 carries no store vector, the NHWC rows
    of 3 channels are adjacent, so the plan loads vectors along h*w and writes
    the output tile flat (the mirror of the odd-plane case)."""
    op = FusedOp(W.cfg3(256, 3, 224, 224), jit=0, autotune=0)
    li = op.info()["launches"][0]
    assert (li["class"], li["width"], li["read_width"]) == ("transpose", 1, 8)
    src = op.source()
    assert "flat tile of TR output rows" in src and "fop::vstore<fop::F16, 8, 16" in src
    op2 = FusedOp(W.nhwc_to_nchw(256, 7, 7, 2048), jit=0, autotune=0)
    assert "flat tile of TR output rows" in op2.source()


def test_min_of_min_and_sum_compiles():
    """CUDA 12.9's NVVM crashed the process (SIGILL inside NVRTC) on
    min(min(a, b), a + b) written with fminf (fuzz seed 15, case 161); the
    device header's min/max are inline PTX.  Compiling it must not kill us."""
    d = {
        "name": "minmin", "loops": {"l0": 24},
        "tensors": {"x0": {"shape": [24], "dtype": "bf16", "role": "in", "init": ("normal", 0.0, 1.0, 1), "strides": [1]},
                    "out": {"shape": [24], "dtype": "bf16", "role": "out", "init": None, "strides": [1]}},
        "stmts": [{"kind": "assign", "loops": ["l0"], "write": ("out", ["l0"]), "reads": [("x0", ["l0"])],
                   "expr": [("load", 0), ("relu", 0), ("add", 0, 1), ("min", 0, 1), ("sub", 0, 0), ("min", 3, 2)]}],
    }
    for fw in (0, 1):   # the vector kernel and the scalar (narrow) form that crashed
        FusedOp(d, force_width=fw) if fw else FusedOp(d)


def test_mirrored_smem_transpose_needs_aligned_input_rows():
    """Fuzz seed 18 case 260: x0[3,128,1] read as x0[l3,l2,l0] into out[.,.,128,3]:
    the input rows along d_r are not 16-byte aligned for every l3, so the
    flat-output shared-memory path must not be chosen (it compiles either way)."""
    d = {"name": "tr_small", "loops": {"l0": 1, "l1": 24, "l2": 128, "l3": 3},
         "tensors": {"x0": {"shape": [3, 128, 1], "dtype": "bf16", "role": "in", "init": ("normal", 0.0, 1.0, 1),
                            "strides": None},
                     "out": {"shape": [1, 24, 128, 3], "dtype": "bf16", "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "assign", "loops": ["l0", "l1", "l2", "l3"], "write": ("out", ["l0", "l1", "l2", "l3"]),
                    "reads": [("x0", ["l3", "l2", "l0"])],
                    "expr": [("load", 0), ("const", 0.5), ("add", 1, 0), ("div", 2, 2), ("cast", 3, "bf16")]}]}
    FusedOp(d)


def test_peel_chosen_for_odd_rows_only():
    """Per-row peel: rows of odd length keep the full vector width; even rows
    plan exactly as before (no shift code)."""
    assert "pe_s" in FusedOp(W.cfg4a(2, 64, 771), jit=0, autotune=0).source()
    assert "pe_s" not in FusedOp(W.cfg4a(2, 64, 768), jit=0, autotune=0).source()
    li = FusedOp(W.N4["vocab_softmax"](R=4, V=50257), jit=0, autotune=0).info()["launches"][0]
    assert (li["class"], li["width"]) == ("row_reduce", 8)


def test_fast_forms_not_ahead_of_add_or_subtract():
    """16-bit fast forms: ÷ invariant as × rcp with a remainder correction
    everywhere; exp/sigmoid approximations only where the value reaches the
    output without an add/sub (fuzz seed 21 case 294)."""
    def op(expr):
        return {"name": "fast", "loops": {"a": 64, "b": 256},
                "tensors": {"x": {"shape": [64, 256], "dtype": "f32", "role": "in", "init": ("normal", 0.0, 1.0, 1),
                                  "strides": None},
                            "y": {"shape": [64, 256], "dtype": "f32", "role": "in", "init": ("normal", 0.0, 1.0, 2),
                                  "strides": None},
                            "out": {"shape": [64, 256], "dtype": "f16", "role": "out", "init": None, "strides": None}},
                "stmts": [{"kind": "assign", "loops": ["a", "b"], "write": ("out", ["a", "b"]),
                           "reads": [("x", ["a", "b"]), ("y", ["a", "b"])], "expr": expr}]}
    # division by an invariant: x * rcp(c) plus one remainder correction, also ahead of an add
    direct = FusedOp(op([("load", 0), ("const", -1.5), ("div", 0, 1)]), jit=0, autotune=0).source()
    summed = FusedOp(op([("load", 0), ("const", -1.5), ("div", 0, 1), ("load", 1), ("add", 2, 3)]),
                     jit=0, autotune=0).source()
    assert "fop::div2_by(" in direct and "fop::div2_by(" in summed
    # exp's fast form only where no add/sub follows
    e_direct = FusedOp(op([("load", 0), ("exp", 0)]), jit=0, autotune=0).source()
    e_summed = FusedOp(op([("load", 0), ("exp", 0), ("load", 1), ("add", 1, 2)]), jit=0, autotune=0).source()
    assert "fop::exp_fast(" in e_direct and "fop::exp_fast(" not in e_summed


def _int_desc(expr, out="i32", xin="i32", kind="assign", write_idx=("i",)):
    t = lambda dt, role, shape=(64,): {"shape": list(shape), "dtype": dt, "role": role, "init": None, "strides": None}  # noqa: E731
    return {"name": "i", "loops": {"i": 64, "k": 4},
            "tensors": {"a": t(xin, "in", (64, 4)), "out": t(out, "out")},
            "stmts": [{"kind": kind, "op": "sum", "loops": ["i", "k"] if kind == "reduce" else ["i"],
                       "write": ("out", list(write_idx)),
                       "reads": [("a", ["i", "k"] if kind == "reduce" else ["i", 0])], "expr": expr}]}


@pytest.mark.parametrize("desc,status", [
    (_int_desc([("load", 0), ("const", 3.0), ("mul", 0, 1), ("neg", 2), ("abs", 3), ("relu", 4)]), None),
    (_int_desc([("load", 0), ("const", 2.0), ("div", 0, 1)]), "FOP_E_INVALID"),          # / not defined on i32
    (_int_desc([("load", 0), ("exp", 0)]), "FOP_E_INVALID"),
    (_int_desc([("load", 0), ("const", 0.5), ("add", 0, 1)]), "FOP_E_INVALID"),          # non-integral constant
    (_int_desc([("load", 0), ("const", 1.0), ("add", 0, 1)], out="f32"), "FOP_E_INVALID"),  # float stmt reads i32
    (_int_desc([("load", 0), ("const", 1.0), ("add", 0, 1)], xin="f32"), "FOP_E_INVALID"),  # int stmt reads f32
    (_int_desc([("load", 0)], out="f32"), "FOP_E_INVALID"),                              # not a move: a conversion
    (_int_desc([("load", 0)]), None),                                                     # pure i32 move
    (_int_desc([("load", 0)], kind="reduce"), None),                                      # i32 column sum
])
def test_integer_statement_rules_match_the_oracle(desc, status):
    """Reading R30: the product accepts exactly the integer statements the oracle defines
    (tests/test_oracle_ops.py), reductions included."""
    from oracle import oracle as O
    x = {"a": np.arange(256, dtype=np.float32 if desc["tensors"]["a"]["dtype"] == "f32" else np.int32)}
    if status is None:
        FusedOp(desc, jit=0)
        O.run(desc, x)
        return
    with pytest.raises(FopError) as e:
        FusedOp(desc, jit=0)
    assert e.value.status == status
    if status == "FOP_E_INVALID":
        with pytest.raises(ValueError):
            O.run(desc, x)


def test_integer_kernels_compile_for_sm100a():
    d = _int_desc([("load", 0), ("const", 3.0), ("mul", 0, 1), ("const", -7.0), ("max", 2, 3)])
    op = FusedOp(d)
    src = op.source()
    assert "fop::imul(" in src and "fop::imax(" in src and "fop::mul2" not in src
    assert "IMAD" in _sass(op.cubin(0)) or "IMUL" in _sass(op.cubin(0))


@pytest.mark.parametrize("R,C,dtype,fold", [(65536, 1001, "f16", True), (777, 1001, "f16", True), (40000, 3, "f16", True),
                                            (5000, 37, "f32", True), (4098, 1002, "f16", True), (4096, 1002, "f16", True),
                                            (65536, 1000, "f16", False), (7, 1001, "f16", False), (3, 1002, "f16", False)])
def test_column_reduction_over_odd_rows_folds_groups_of_rows(R, C, dtype, fold):
    """COL_REDUCE over dense rows no vector divides: with R >= P = W / gcd(C, W) the kernel
    reads the first R - R mod P rows as [R/P, P*C] with aligned full vectors and folds P wide
    columns per output (workspace holds the P*C sums), the R mod P tail rows added
    element-wise by the folding block; fewer rows than P (or C divisible by W): no fold."""
    import math
    d = {"name": "colred", "loops": {"r": R, "c": C},
         "tensors": {"x": {"shape": [R, C], "dtype": dtype, "role": "in", "init": ("normal", 0.0, 1.0, 71), "strides": None},
                     "out": {"shape": [C], "dtype": "f32", "role": "out", "init": None, "strides": None}},
         "stmts": [{"kind": "reduce", "op": "sum", "loops": ["r", "c"], "write": ("out", ["c"]),
                    "reads": [("x", ["r", "c"])], "expr": [("load", 0)]}]}
    op = FusedOp(d, jit=0, autotune=0)
    src, li = op.source(), op.info()["launches"][0]
    assert li["class"] == "col_reduce" and li["width"] == 16 // (4 if dtype == "f32" else 2)
    assert ("fold_flag" in src) == fold
    if fold:
        P = li["width"] // math.gcd(C, li["width"])
        assert f"q = rr * {P}u" in src and f"c_ < {C}u" in src
        assert ("tr_ < " in src) == (R % P != 0)
        assert op.info()["workspace_bytes"] >= P * C * 4


def test_narrow_variant_source_is_inspectable():
    """fop_plan_source(plan, -1 - k, ...) returns launch k's narrow variant (the kernel run for
    base pointers off the planned alignment): scalar accesses, its own kernel name, and for a
    TMA-planned transpose no tensor-map path (fuzz seed 41)."""
    op = FusedOp(W.cfg3(2, 64, 8, 8), jit=0, autotune=0)
    assert "TRANSPOSE via TMA" in op.source(0)
    nsrc = op.source(0, narrow=True)
    assert "_narrow" in nsrc and "TMA" not in nsrc and "tma_load" not in nsrc
    with pytest.raises(Exception):
        op.source(-5)
