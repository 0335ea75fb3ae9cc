"""Transposes beyond cfg3: dtypes, channel counts, the reverse direction and a
plain 2-D transpose, each timed like tools/sweep.py (rotating copies > 3x L2,
batches of back-to-back launches, auto-tuned geometry) next to a device copy of
the same bytes.  Prints one JSON line per case.

    python tools/tr_variety.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from bench import to_device  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402

L2 = 126 << 20


CASES = [
    ("cfg3 f16 [256,256,56,56]", lambda: W.cfg3()),
    ("cfg3 bf16 [256,256,56,56]", lambda: W.cfg3(dtype="bf16")),
    ("cfg3 f32 [128,256,56,56]", lambda: W.cfg3(N=128, dtype="f32")),
    ("NCHW->NHWC f16 C=64 [128,64,112,112]", lambda: W.cfg3(128, 64, 112, 112)),
    ("NCHW->NHWC f16 C=96 [256,96,56,56]", lambda: W.cfg3(256, 96, 56, 56)),
    ("NCHW->NHWC f16 C=3 [256,3,224,224]", lambda: W.cfg3(256, 3, 224, 224)),
    ("NCHW->NHWC f16 C=2048 [256,2048,7,7]", lambda: W.cfg3(256, 2048, 7, 7)),
    ("NHWC->NCHW f16 [256,56,56,256]", lambda: W.nhwc_to_nchw(256, 56, 56, 256)),
    ("NHWC->NCHW f16 7x7 [256,7,7,2048]", lambda: W.nhwc_to_nchw(256, 7, 7, 2048)),
    ("2-D f32 [16384,16384]", lambda: W.transpose2d(16384, 16384, "f32")),
    ("2-D f16 [8192,24576]", lambda: W.transpose2d(8192, 24576, "f16")),
    ("NHWC->NCHW f16 [256,7,9,64] (H*W=63)", lambda: W.nhwc_to_nchw(256, 7, 9, 64)),
]


def time_op(run, sets, n=20, reps=5):
    """Graph-replayed batches, as in tools/red_variety.py (one timing method for every sweep)."""
    import importlib.util
    spec = importlib.util.spec_from_file_location("red_variety", os.path.join(ROOT, "tools", "red_variety.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m.time_op(run, sets, n, reps)


def main():
    for name, mk in CASES:
        d = mk()
        try:
            op = FusedOp(d)
        except Exception as ex:  # noqa: BLE001
            print(json.dumps({"case": name, "error": str(ex)[:200]}), flush=True)
            continue
        nbytes = W.algorithmic_bytes(d)
        copies = max(1, min(8, -(-3 * L2 // nbytes)))
        x = W.make_inputs(d)
        o = W.alloc_outputs(d, fill_nan=False)
        sets = [{n: to_device(x[n] if t["role"] == "in" else o[n], t["dtype"], "cuda")
                 for n, t in d["tensors"].items() if t["role"] != "temp"} for _ in range(copies)]
        ms = time_op(lambda s: op.run(s), sets)
        half = nbytes // 2
        src = [torch.empty(half, dtype=torch.uint8, device="cuda") for _ in range(copies)]
        dst = [torch.empty(half, dtype=torch.uint8, device="cuda") for _ in range(copies)]
        cms = time_op(lambda k: dst[k].copy_(src[k]), list(range(copies)))
        li = op.info()["launches"][0]
        print(json.dumps({"case": name, "class": li["class"], "vec_loop": li["vec_loop"], "width": li["width"],
                          "read_loop": li["read_loop"], "read_width": li["read_width"],
                          "selected": list(op.selected(0)), "us": ms * 1e3, "GB_s": nbytes / ms / 1e6,
                          "copy_GB_s": nbytes / cms / 1e6, "frac_of_copy": cms / ms}), flush=True)
        del sets, src, dst
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
