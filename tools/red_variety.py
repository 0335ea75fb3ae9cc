"""Reductions beyond cfg4a/cfg4b: row and column sums of other shapes and
dtypes, each timed like tools/sweep.py (rotating copies > 3x L2, batches of
back-to-back launches, auto-tuned geometry) next to a device READ of the same
input bytes (the reductions' traffic is the input read).  One JSON line per case.

    python tools/red_variety.py
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


def rowsum(R, C, dtype="f16"):
    return {
        "name": "rowsum", "loops": {"r": R, "c": C},
        "tensors": {"x": {"shape": [R, C], "dtype": dtype, "role": "in", "init": ("normal", 0.0, 1.0, 5),
                          "strides": None},
                    "out": {"shape": [R], "dtype": "f32", "role": "out", "init": None, "strides": None}},
        "stmts": [{"kind": "reduce", "op": "sum", "loops": ["r", "c"], "write": ("out", ["r"]),
                   "reads": [("x", ["r", "c"])], "expr": [("load", 0)]}],
    }


def colsum(R, C, dtype="f16"):
    d = W.cfg4b(R, C)
    d["tensors"]["x"]["dtype"] = dtype
    return d


CASES = [
    ("colsum f16 [65536,1024] (cfg4b)", lambda: W.cfg4b()),
    ("colsum f32 [4194304,16]", lambda: colsum(4194304, 16, "f32")),
    ("colsum f16 [512,131072]", lambda: colsum(512, 131072)),
    ("colsum f32 [8192,4096]", lambda: colsum(8192, 4096, "f32")),
    ("rowsum f16 [65536,1024]", lambda: rowsum(65536, 1024)),
    ("rowsum f16 [1048576,64]", lambda: rowsum(1048576, 64)),
    ("rowsum f32 [4194304,16]", lambda: rowsum(4194304, 16, "f32")),
    ("rowsum f16 [64,1048576]", lambda: rowsum(64, 1048576)),
    ("rowsum f32 [8192,4096]", lambda: rowsum(8192, 4096, "f32")),
    ("rowsum f16 [100,524288]", lambda: rowsum(100, 524288)),
    ("rowsum f32 [32,1048576]", lambda: rowsum(32, 1048576, "f32")),
    ("vocab softmax f16 [256,32000]", lambda: W.N4["vocab_softmax"](R=256, V=32000)),
    ("vocab softmax f16 [256,50257] (odd)", lambda: W.N4["vocab_softmax"](R=256, V=50257)),
    ("layernorm f16 [16384,1023] (odd)", lambda: dict(W.N4["bert_layernorm"](B=32, S=512, H=1023), name="ln_odd")),
    ("layernorm f16 [16384,1024]", lambda: dict(W.N4["bert_layernorm"](B=32, S=512, H=1024), name="ln")),
]


def time_op(run, sets, n=20, reps=5):
    """Median per-launch ms over `reps` batches of `n` launches rotating over `sets`.
    The batch is captured once in a CUDA graph and replayed, so a small operator is
    timed on the device rather than by the host's per-call launch cost (eager
    launches if the capture fails)."""
    import statistics
    for i in range(3):
        run(sets[i % len(sets)])
    torch.cuda.synchronize()
    batch = lambda: [run(sets[i % len(sets)]) for i in range(n)]  # noqa: E731
    try:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            batch()
        g.replay()
        torch.cuda.synchronize()
        batch = g.replay
    except Exception:   # not capturable: eager launches
        torch.cuda.synchronize()
    per = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        batch()
        e.record()
        torch.cuda.synchronize()
        per.append(s.elapsed_time(e) / n)
    return statistics.median(per)


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
        xin = [n for n, t in d["tensors"].items() if t["role"] == "in"][0]
        src = [s[xin].view(torch.uint8).reshape(-1) for s in sets]
        rms = time_op(lambda k: torch.sum(src[k][: src[k].numel() // 4].view(torch.int32), dtype=torch.int64),
                      list(range(copies)))
        li = op.info()["launches"]
        print(json.dumps({"case": name, "classes": [q["class"] for q in li], "selected": list(op.selected(0)),
                          "us": ms * 1e3, "GB_s": nbytes / ms / 1e6,
                          "torch_sum_read_GB_s": x[xin].nbytes / rms / 1e6}), flush=True)
        del sets, src
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
