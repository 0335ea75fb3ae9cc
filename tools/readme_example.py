"""The README usage example, runnable: python tools/readme_example.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp

# LayerNorm-style statistics fused with a bias + GELU producer, [B*S, H] fp16:
#   y[r,h] = f16(gelu(x[r,h] + b[h]));  mean[r] = sum_h y[r,h] / H
R, H = 32768, 768
desc = {
    "name": "bias_gelu_mean",
    "loops": {"r": R, "h": H},
    "tensors": {
        "x": {"shape": [R, H], "dtype": "f16", "role": "in"},
        "b": {"shape": [H], "dtype": "f16", "role": "in"},
        "y": {"shape": [R, H], "dtype": "f16", "role": "out"},
        "mean": {"shape": [R], "dtype": "f32", "role": "out"},
    },
    "stmts": [
        {"kind": "assign", "loops": ["r", "h"], "write": ("y", ["r", "h"]),
         "reads": [("x", ["r", "h"]), ("b", ["h"])],
         "expr": [("load", 0), ("load", 1), ("add", 0, 1), ("gelu_tanh", 2)]},
        {"kind": "reduce", "op": "sum", "loops": ["r", "h"], "write": ("mean", ["r"]),
         "reads": [("y", ["r", "h"])], "expr": [("load", 0)],
         "finalize": [("acc",), ("const", float(H)), ("div", 0, 1)]},
    ],
}
op = FusedOp(desc)                 # plan (Algorithm 2) + generate + NVRTC-compile for sm_100a
print(op.info()["launches"])      # kernel class, vector loop and width, grid
if torch.cuda.is_available():
    t = {"x": torch.randn(R, H, device="cuda").half(), "b": torch.randn(H, device="cuda").half(),
         "y": torch.empty(R, H, device="cuda", dtype=torch.half), "mean": torch.empty(R, device="cuda")}
    op.run(t)                      # enqueued on torch's current stream
