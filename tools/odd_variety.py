"""Odd extents across the classes (vector loops that do not divide): timed like
tools/sweep.py; one JSON line per case."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import importlib.util  # noqa: E402


def _load(name):
    spec = importlib.util.spec_from_file_location(name, os.path.join(ROOT, "tools", name + ".py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


rv, ev = _load("red_variety"), _load("ew_variety")
import torch  # noqa: E402
import workloads as W  # noqa: E402
from bench import to_device  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402

CASES = [
    ("colsum f16 [65536,1001]", lambda: rv.colsum(65536, 1001)),
    ("colsum f16 [65536,1000]", lambda: rv.colsum(65536, 1000)),
    ("rowsum f16 [65536,1001]", lambda: rv.rowsum(65536, 1001)),
    ("bias add f16 [65536,1001]", lambda: ev.binop([65536, 1001], "f16", bshape=[1001], bidx=["l1"])),
    ("NCHW->NHWC f16 C=255 [128,255,56,56]", lambda: W.cfg3(128, 255, 56, 56)),
    ("NCHW->NHWC f16 C=3 [256,3,224,224]", lambda: W.cfg3(256, 3, 224, 224)),
    ("NHWC->NCHW f16 7x7 [256,7,7,2048]", lambda: W.nhwc_to_nchw(256, 7, 7, 2048)),
    ("NHWC->NCHW f16 [256,7,9,64] (H*W=63)", lambda: W.nhwc_to_nchw(256, 7, 9, 64)),
]
for name, mk in CASES:
    d = mk()
    op = FusedOp(d)
    nbytes = W.algorithmic_bytes(d)
    copies = max(1, min(8, -(-3 * rv.L2 // nbytes)))
    x = W.make_inputs(d)
    o = W.alloc_outputs(d, fill_nan=False)
    sets = [{n: to_device(x[n] if t["role"] == "in" else o[n], t["dtype"], "cuda")
             for n, t in d["tensors"].items() if t["role"] != "temp"} for _ in range(copies)]
    ms = rv.time_op(lambda s: op.run(s), sets)
    li = op.info()["launches"][0]
    print(json.dumps({"case": name, "class": li["class"], "width": li["width"], "selected": list(op.selected(0)),
                      "us": ms * 1e3, "GB_s": nbytes / ms / 1e6}), flush=True)
    del sets
    torch.cuda.empty_cache()
