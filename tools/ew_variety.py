"""Elementwise operators beyond cfg2: layouts, broadcasts, padded strides,
casts, odd sizes, each timed like tools/sweep.py (rotating copies > 3x L2,
batches of back-to-back launches, auto-tuned geometry) next to a device copy
of the same bytes.  One JSON line per case.

    python tools/ew_variety.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import importlib.util  # noqa: E402

spec = importlib.util.spec_from_file_location("rv", os.path.join(ROOT, "tools", "red_variety.py"))
rv = importlib.util.module_from_spec(spec)
spec.loader.exec_module(rv)
import torch  # noqa: E402

import workloads as W  # noqa: E402
from bench import to_device  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402


def T(shape, dtype, role, strides=None, seed=1):
    return {"shape": list(shape), "dtype": dtype, "role": role,
            "init": ("uniform", -1.0, 1.0, seed) if role == "in" else None, "strides": strides}


def binop(shape, dtype="f16", op="add", out_dtype=None, bshape=None, bidx=None, strides=None):
    loops = {f"l{i}": e for i, e in enumerate(shape)}
    names = list(loops)
    return {
        "name": "binop", "loops": loops,
        "tensors": {"a": T(shape, dtype, "in", strides, 1),
                    "b": T(bshape or shape, dtype, "in", None, 2),
                    "out": T(shape, out_dtype or dtype, "out")},
        "stmts": [{"kind": "assign", "loops": names, "write": ("out", names),
                   "reads": [("a", names), ("b", bidx or names)],
                   "expr": [("load", 0), ("load", 1), (op, 0, 1)]}],
    }


def cast(shape, src, dst):
    loops = {f"l{i}": e for i, e in enumerate(shape)}
    names = list(loops)
    return {"name": "cast", "loops": loops,
            "tensors": {"a": T(shape, src, "in"), "out": T(shape, dst, "out")},
            "stmts": [{"kind": "assign", "loops": names, "write": ("out", names),
                       "reads": [("a", names)], "expr": [("load", 0)]}]}


CASES = [
    ("cfg2 BN+ReLU+cast NCHW", lambda: W.cfg2()),
    ("BN+ReLU+cast NHWC [128,112,112,64]", lambda: W.cfg2_nhwc()),
    ("residual add f16 [128,256,56,56]", lambda: binop([128, 256, 56, 56])),
    ("bias add f32 [65536,1000]", lambda: binop([65536, 1000], "f32", bshape=[1000], bidx=["l1"])),
    ("bias add f32 [65536,1001] (odd)", lambda: binop([65536, 1001], "f32", bshape=[1001], bidx=["l1"])),
    ("row scale f16 [65536,1024]*s[r]", lambda: binop([65536, 1024], "f16", "mul", bshape=[65536], bidx=["l0"])),
    ("padded rows f16 [65536,1000] pitch 1024", lambda: binop([65536, 1000], "f16", strides=[1024, 1])),
    ("cast f32->bf16 [268435456]", lambda: cast([268435456], "f32", "bf16")),
    ("cast f16->f32 [134217728]", lambda: cast([134217728], "f16", "f32")),
]


def main():
    for name, mk in CASES:
        d = mk()
        try:
            op = FusedOp(d, autotune=int(os.environ.get("FOP_SWEEP_AUTOTUNE", "1")))
        except Exception as ex:  # noqa: BLE001
            print(json.dumps({"case": name, "error": str(ex)[:300]}), flush=True)
            continue
        nbytes = W.algorithmic_bytes(d)
        copies = max(1, min(8, -(-3 * rv.L2 // nbytes)))
        x = W.make_inputs(d)
        o = W.alloc_outputs(d, fill_nan=False)
        sets = [{n: to_device(x[n] if t["role"] == "in" else o[n], t["dtype"], "cuda")
                 for n, t in d["tensors"].items() if t["role"] != "temp"} for _ in range(copies)]
        ms = rv.time_op(lambda s: op.run(s), sets)
        half = nbytes // 2
        src = [torch.empty(half, dtype=torch.uint8, device="cuda") for _ in range(copies)]
        dst = [torch.empty(half, dtype=torch.uint8, device="cuda") for _ in range(copies)]
        cms = rv.time_op(lambda k: dst[k].copy_(src[k]), list(range(copies)))
        li = op.info()["launches"][0]
        print(json.dumps({"case": name, "class": li["class"], "vec_loop": li["vec_loop"], "width": li["width"],
                          "selected": list(op.selected(0)), "us": ms * 1e3, "GB_s": nbytes / ms / 1e6,
                          "copy_GB_s": nbytes / cms / 1e6, "frac_of_copy": cms / ms}), flush=True)
        del sets, src, dst
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
