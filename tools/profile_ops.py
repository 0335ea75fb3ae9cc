"""Run each fused operator of the bench suite a few times (for ncu).

    ncu --set full --clock-control none --import-source on --profile-from-start off \
        -k regex:fop_ -c 4 -o gpurun_out/prof python tools/profile_ops.py --reps 1

Every op runs twice first (auto-tuning and module loads happen there), then
the profiler is started (cudaProfilerStart) and each op runs `--reps` times
with the geometry the tuner kept, so `-c 4` captures one launch per kernel.
Extra flags forward planner options (--vec-bytes, --order) for ablations.
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from bench import OPS, to_device  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--ops", default="cfg2,cfg3,cfg4a,cfg4b")
    ap.add_argument("--vec-bytes", type=int, default=0)
    ap.add_argument("--order", default=None)
    ap.add_argument("--force-width", type=int, default=0)
    a = ap.parse_args()
    opts = {}
    if a.vec_bytes:
        opts["max_vec_bytes"] = a.vec_bytes
    if a.order:
        opts["coalesce_order"] = a.order
    if a.force_width:
        opts["force_width"] = a.force_width
    want = a.ops.split(",")
    ops = []
    for name, mk, cls in OPS:
        if name not in want:
            continue
        d = mk()
        op = FusedOp(d, **opts)
        x = W.make_inputs(d)
        o = W.alloc_outputs(d, fill_nan=False)
        tens = {n: to_device(x[n] if t["role"] in ("in", "inout") else o[n], t["dtype"], "cuda")
                for n, t in d["tensors"].items() if t["role"] != "temp"}
        ops.append((name, op, tens))
    for name, op, tens in ops:          # first runs: auto-tuning candidates, module loads
        op.run(tens)
        op.run(tens)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStart()   # ncu --profile-from-start off: capture from here
    for _ in range(a.reps):
        for name, op, tens in ops:
            op.run(tens)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStop()
    print("done", [(n, op.selected(0)) for n, op, _ in ops])


if __name__ == "__main__":
    main()
