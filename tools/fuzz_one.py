"""Re-run one fuzz case (seed, index) with the campaign's checks (crash triage).
    python -X faulthandler tools/fuzz_one.py SEED INDEX [--no-repeat] [--steps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import numpy as np  # noqa: E402
from fuzz_gen import random_op  # noqa: E402
import fuzz_campaign as F  # noqa: E402

seed, idx = int(sys.argv[1]), int(sys.argv[2])
rng = np.random.default_rng(seed)
for _ in range(idx + 1):
    d = random_op(rng)
print(d, flush=True)
if "--steps" in sys.argv:
    import torch
    import workloads as W
    from harness import run_gpu, device_tensors
    x = W.make_inputs(d)
    opts = {"autotune": 0} if "--no-tune" in sys.argv else {}
    got, op = run_gpu(d, x, **opts)
    print("first run ok", op.selected(0), flush=True)
    for off in (0, 1, 0, 1):
        dev = device_tensors(d, x, offset=off)
        print("run offset", off, [hex(t.data_ptr()) for t in dev.values()], flush=True)
        op.run(dev)
        torch.cuda.synchronize()
        print("  ok", flush=True)
else:
    print(F.check(d, "--no-repeat" not in sys.argv), flush=True)
print("ok", flush=True)
