"""Few long rows (rows < SMs): time the ROW_REDUCE cluster geometry variants
(CTAs per row Q, warps per row G, blocks/SM) on row sums like [64, 1048576]."""
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

VARIANTS = ["", "FOP_ROW_Q=8", "FOP_ROW_Q=8,FOP_ROW_MINB=4", "FOP_ROW_Q=8,FOP_ROW_G=4", "FOP_ROW_Q=8,FOP_ROW_G=16",
            "FOP_ROW_Q=4,FOP_ROW_G=16", "FOP_ROW_Q=8,FOP_ROW_ROU=4"]
for R, C, dt in [(64, 1048576, "f16"), (32, 1048576, "f32"), (100, 524288, "f16")]:
    d = rv.rowsum(R, C, dt)
    nbytes = W.algorithmic_bytes(d)
    copies = max(1, min(8, -(-3 * rv.L2 // nbytes)))
    x = W.make_inputs(d)
    o = W.alloc_outputs(d, fill_nan=False)
    sets = [{n: to_device(x[n] if t["role"] == "in" else o[n], t["dtype"], "cuda")
             for n, t in d["tensors"].items() if t["role"] != "temp"} for _ in range(copies)]
    for v in VARIANTS:
        env = dict(kv.split("=") for kv in v.split(",") if kv)
        os.environ.update(env)
        try:
            op = FusedOp(d, autotune=0)
            ms = rv.time_op(lambda s: op.run(s), sets)
            li = op.info()["launches"][0]
            print(json.dumps({"shape": [R, C, dt], "variant": v, "grid": li["grid"], "block": li["block"],
                              "us": ms * 1e3, "GB_s": nbytes / ms / 1e6}), flush=True)
        except Exception as e:  # noqa: BLE001
            print(json.dumps({"shape": [R, C, dt], "variant": v, "error": str(e)[:200]}), flush=True)
        for k in env:
            del os.environ[k]
    del sets
    torch.cuda.empty_cache()
