"""Time one fused operator under several planner/geometry variants.

    python tools/sweep.py cfg2 "FOP_EW_U=2,FOP_EW_MINB=4" "FOP_EW_U=4,FOP_EW_MINB=3" ...
    python tools/sweep.py cfg3 "opt:max_vec_bytes=32" "opt:coalesce_order=memory"

Each variant: plan under the given env knobs / plan options, 5 warm-up runs,
then 30 timed runs (CUDA events around the launch on the current stream),
L2 flushed (256 MiB memset) before every timed run.  Prints median/min GB/s
(algorithmic bytes) per variant, one JSON line each.
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from bench import to_device  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402


def main():
    name = sys.argv[1]
    variants = sys.argv[2:] or [""]
    d = W.CONFIGS[name]()
    x = W.make_inputs(d)
    o = W.alloc_outputs(d, fill_nan=False)
    tens = {n: to_device(x[n] if t["role"] in ("in", "inout") else o[n], t["dtype"], "cuda")
            for n, t in d["tensors"].items() if t["role"] != "temp"}
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    nbytes = W.algorithmic_bytes(d)
    for v in variants:
        env, opts = {}, {}
        for kv in filter(None, v.split(",")):
            k, val = kv.split("=")
            if k.startswith("opt:"):
                opts[k[4:]] = val if not val.lstrip("-").isdigit() else int(val)
            else:
                env[k] = val
        old = {k: os.environ.get(k) for k in env}
        os.environ.update(env)
        try:
            op = FusedOp(d, **opts)
        except Exception as e:
            print(json.dumps({"op": name, "variant": v, "error": str(e)[:300]}), flush=True)
            continue
        finally:
            for k, val in old.items():
                if val is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = val
        for _ in range(5):
            op.run(tens)
        times = []
        for _ in range(30):
            flush.zero_()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            op.run(tens)
            e.record()
            torch.cuda.synchronize()
            times.append(s.elapsed_time(e))
        med = statistics.median(times)
        li = op.info()["launches"][0]
        print(json.dumps({"op": name, "variant": v, "us_median": med * 1e3, "us_min": min(times) * 1e3,
                          "GBs_median": nbytes / med / 1e6, "GBs_best": nbytes / min(times) / 1e6,
                          "grid": li["grid"], "class": li["class"], "width": li["width"]}), flush=True)


if __name__ == "__main__":
    main()
