"""Python wrapper of the C oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline
leg and ``--impl reference``) may import this module.  It parses the workload
dict form with its own code (no import of the product package) and fills the
oracle's own C structs (``fop_oracle.h``).

``run(desc, inputs)`` evaluates the fused operator in the original program
order and returns every non-input tensor as a flat numpy
buffer (``workloads.inputs`` layout).
"""

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "liboracle.so")
SRC = os.path.join(HERE, "fop_oracle.c")

RANK, LOOPS, READS, NODES = 8, 8, 8, 64
ELEM = {"f32": 0, "f16": 1, "bf16": 2, "i32": 3}
NP = {"f32": np.float32, "f16": np.float16, "bf16": np.uint16, "i32": np.int32}
KIND = {"load": 1, "const": 2, "acc": 3, "add": 4, "sub": 5, "mul": 6, "div": 7,
        "max": 8, "min": 9, "neg": 10, "abs": 11, "sqrt": 12, "relu": 13,
        "exp": 14, "log": 15, "tanh": 16, "sigmoid": 17, "gelu_tanh": 18,
        "gelu_erf": 19, "cast": 20}


class Array(C.Structure):
    _fields_ = [("data", C.c_void_p), ("elem", C.c_int), ("rank", C.c_int),
                ("shape", C.c_longlong * RANK), ("stride", C.c_longlong * RANK)]


class Ref(C.Structure):
    _fields_ = [("array", C.c_int), ("iter", C.c_int * RANK), ("off", C.c_longlong * RANK)]


class Node(C.Structure):
    _fields_ = [("kind", C.c_int), ("x", C.c_int), ("y", C.c_int), ("elem", C.c_int),
                ("c", C.c_double)]


class Statement(C.Structure):
    _fields_ = [("reduce", C.c_int), ("reduce_max", C.c_int), ("nloops", C.c_int),
                ("loops", C.c_int * LOOPS), ("target", Ref), ("nreads", C.c_int),
                ("reads", Ref * READS), ("nnodes", C.c_int), ("nodes", Node * NODES),
                ("nfin", C.c_int), ("fin", Node * NODES)]


def build(force=False):
    """Compile liboracle.so (plain C, -O2, no FP contraction, no fast math)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-D_GNU_SOURCE", "-ffp-contract=off",
                               "-fno-fast-math", "-fPIC", "-shared", "-o", LIB, SRC, "-lm"])
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = C.CDLL(LIB)
        _lib.orc_run.restype = C.c_int
        _lib.orc_f32_to_f16.restype = C.c_uint16
        _lib.orc_f32_to_f16.argtypes = [C.c_float]
        _lib.orc_f16_to_f32.restype = C.c_float
        _lib.orc_f16_to_f32.argtypes = [C.c_uint16]
        _lib.orc_f32_to_bf16.restype = C.c_uint16
        _lib.orc_f32_to_bf16.argtypes = [C.c_float]
        _lib.orc_bf16_to_f32.restype = C.c_float
        _lib.orc_bf16_to_f32.argtypes = [C.c_uint16]
        _lib.orc_gelu_tanh.restype = C.c_float
        _lib.orc_gelu_tanh.argtypes = [C.c_float]
    return _lib


def _strides(t):
    if t.get("strides"):
        return list(t["strides"])
    st, acc = [], 1
    for s in reversed(t["shape"]):
        st.append(acc)
        acc *= s
    return list(reversed(st))


def _span(t):
    if any(s == 0 for s in t["shape"]):
        return 0
    return 1 + sum((s - 1) * abs(k) for s, k in zip(t["shape"], _strides(t)))


def _ref(acc, loop_id, tensor_id):
    name, index = acc
    r = Ref()
    r.array = tensor_id[name]
    for d in range(RANK):
        r.iter[d] = -1
        r.off[d] = 0
    for d, e in enumerate(index):
        if isinstance(e, str):
            r.iter[d] = loop_id[e]
        elif isinstance(e, (tuple, list)):
            r.iter[d] = loop_id[e[0]]
            r.off[d] = int(e[1])
        else:
            r.off[d] = int(e)
    return r


def _node(spec):
    n = Node()
    n.kind = KIND[spec[0]]
    n.x = n.y = -1
    n.elem = 0
    n.c = 0.0
    op = spec[0]
    if op == "load":
        n.x = int(spec[1])
    elif op == "const":
        n.c = float(np.float32(spec[1]))
    elif op == "acc":
        pass
    elif op == "cast":
        n.x = int(spec[1])
        n.elem = ELEM[spec[2]]
    elif op in ("add", "sub", "mul", "div", "max", "min"):
        n.x, n.y = int(spec[1]), int(spec[2])
    else:
        n.x = int(spec[1])
    return n


def run(desc, inputs, outputs=None, stmts=None):
    """Evaluate ``desc`` on ``inputs`` (name -> flat buffer).

    Returns name -> flat buffer for every OUT / INOUT / TEMP tensor.
    ``outputs`` may pre-supply output buffers (e.g. NaN-filled);
    ``stmts`` optionally restricts execution to a prefix/subset (indices).
    """
    L = lib()
    loops = list(desc["loops"].keys())
    loop_id = {n: i for i, n in enumerate(loops)}
    names = list(desc["tensors"].keys())
    tensor_id = {n: i for i, n in enumerate(names)}
    bufs = {}
    arrays = (Array * len(names))()
    for i, n in enumerate(names):
        t = desc["tensors"][n]
        if t["role"] == "in":
            buf = np.ascontiguousarray(inputs[n])
        elif t["role"] == "inout":
            buf = np.array(inputs[n], copy=True)
        elif outputs is not None and n in outputs:
            buf = outputs[n]
        else:
            buf = np.zeros(max(1, _span(t)), NP[t["dtype"]])
        assert buf.dtype == NP[t["dtype"]], (n, buf.dtype, t["dtype"])
        assert buf.size >= _span(t), (n, buf.size, _span(t))
        bufs[n] = buf
        a = arrays[i]
        a.data = buf.ctypes.data
        a.elem = ELEM[t["dtype"]]
        a.rank = len(t["shape"])
        st = _strides(t)
        for d in range(len(t["shape"])):
            a.shape[d] = t["shape"][d]
            a.stride[d] = st[d]
    sel = range(len(desc["stmts"])) if stmts is None else stmts
    sts = (Statement * max(1, len(desc["stmts"])))()
    for k, si in enumerate(sel):
        s = desc["stmts"][si]
        st = sts[k]
        st.reduce = 1 if s["kind"] == "reduce" else 0
        st.reduce_max = 1 if s.get("op", "sum") == "max" else 0
        st.nloops = len(s["loops"])
        for j, l in enumerate(s["loops"]):
            st.loops[j] = loop_id[l]
        st.target = _ref(s["write"], loop_id, tensor_id)
        st.nreads = len(s["reads"])
        for j, r in enumerate(s["reads"]):
            st.reads[j] = _ref(r, loop_id, tensor_id)
        st.nnodes = len(s["expr"])
        for j, e in enumerate(s["expr"]):
            st.nodes[j] = _node(e)
        fin = s.get("finalize") or []
        st.nfin = len(fin)
        for j, e in enumerate(fin):
            st.fin[j] = _node(e)
    ext = (C.c_longlong * LOOPS)(*[desc["loops"][n] for n in loops])
    err = C.create_string_buffer(512)
    rc = L.orc_run(C.c_int(len(loops)), ext, C.c_int(len(names)), arrays,
                   C.c_int(len(list(sel))), sts, err, C.c_int(512))
    if rc != 0:
        raise ValueError("oracle rejected the descriptor: " + err.value.decode())
    return {n: bufs[n] for n in names if desc["tensors"][n]["role"] != "in"}


def f32_to_f16_bits(v):
    return lib().orc_f32_to_f16(float(v))


def f16_bits_to_f32(h):
    return lib().orc_f16_to_f32(int(h))
