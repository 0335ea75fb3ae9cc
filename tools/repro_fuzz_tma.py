import json, os, sys, traceback
sys.path.insert(0, "tests"); sys.path.insert(0, ".")
import numpy as np, torch
import workloads as W
from harness import device_tensors, to_host
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
d = json.load(open("tests/fuzz_regressions/tma_seed41_case273.json"))
x = W.make_inputs(d)
op = FusedOp(d)
print(op.info()["launches"])
for off in (0, 0, 1, 0, 1, 0):
    dev = device_tensors(d, x, offset=off)
    print("run off", off, {n: hex(t.data_ptr()) for n, t in dev.items()}, flush=True)
    try:
        op.run(dev); torch.cuda.synchronize(); print("  ok selected", op.selected(0), flush=True)
    except Exception as e:
        print("  FAIL", e, flush=True)
