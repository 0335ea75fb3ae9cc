"""Time one fused operator under several planner/geometry variants.

    python tools/sweep.py cfg2 "FOP_EW_U=2,FOP_EW_MINB=4" "FOP_EW_U=4,FOP_EW_MINB=3" ...
    python tools/sweep.py cfg3 "opt:max_vec_bytes=32" "opt:coalesce_order=memory"

Timing: R copies of every tensor (R chosen so the copies exceed 3x the 126 MB
L2), 5 warm-up launches, then 5 batches of 40 launches rotating over the
copies, each batch bracketed by CUDA events on the current stream (event
resolution is ~2 us, too coarse for one 20-40 us launch).  Per-launch time =
batch time / 40; reported: median and best batch, GB/s of algorithmic bytes.
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

L2 = 126 << 20


def main():
    name = sys.argv[1]
    variants = sys.argv[2:] or [""]
    d = (W.CONFIGS.get(name) or W.N4.get(name) or W.ODD.get(name) or W.N3[name])()
    x = W.make_inputs(d)
    o = W.alloc_outputs(d, fill_nan=False)
    nbytes = W.algorithmic_bytes(d)
    copies = max(1, min(16, -(-3 * L2 // nbytes)))
    sets = []
    for _ in range(copies):
        sets.append({n: to_device(x[n] if t["role"] in ("in", "inout") else o[n], t["dtype"], "cuda")
                     for n, t in d["tensors"].items() if t["role"] != "temp"})
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
        def restore():
            for k, val in old.items():
                if val is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = val
        try:
            op = FusedOp(d, **opts)
        except Exception as e:
            restore()
            print(json.dumps({"op": name, "variant": v, "error": str(e)[:300]}), flush=True)
            continue
        # run-time knobs (FOP_TUNE_HOT, ...) stay set until the variant is timed
        for i in range(5):
            op.run(sets[i % copies])
        torch.cuda.synchronize()
        per = []
        n = 40
        for _ in range(5):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for i in range(n):
                op.run(sets[i % copies])
            e.record()
            torch.cuda.synchronize()
            per.append(s.elapsed_time(e) / n)
        med = statistics.median(per)
        restore()
        li = op.info()["launches"][0]
        sel = op.selected(0)
        print(json.dumps({"op": name, "variant": v, "us_median": med * 1e3, "us_min": min(per) * 1e3,
                          "GBs_median": nbytes / med / 1e6, "GBs_best": nbytes / min(per) / 1e6,
                          "grid": li["grid"], "class": li["class"], "width": li["width"], "copies": copies,
                          "selected": list(sel)}),
              flush=True)


if __name__ == "__main__":
    main()
