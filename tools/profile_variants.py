"""Run the session-3 kernel variants once each (after tuning) for ncu:
shared-memory transposes (flat input / flat output tiles), NHWC->NCHW,
short-row and peeled ROW, vector-loop tables (NHWC BN).

    ncu --set full --clock-control none --profile-from-start off -k regex:fop_ -c 7 \
        -o gpurun_out/prof_variants python tools/profile_variants.py
"""
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

CASES = [
    ("tr_smem_in 2048x7x7", lambda: W.cfg3(256, 2048, 7, 7)),
    ("tr_smem_out C=3", lambda: W.cfg3(256, 3, 224, 224)),
    ("nhwc_to_nchw", lambda: W.nhwc_to_nchw(256, 56, 56, 256)),
    ("row_short [1048576,64]", lambda: rv.rowsum(1048576, 64)),
    ("row_peel vocab 50257", lambda: W.N4["vocab_softmax"](R=256, V=50257)),
    ("row_peel layernorm 1023", lambda: dict(W.N4["bert_layernorm"](B=32, S=512, H=1023), name="ln_odd")),
    ("ew_vec_table NHWC BN", lambda: W.cfg2_nhwc()),
]
ops = []
for name, mk in CASES:
    d = mk()
    op = FusedOp(d)
    x = W.make_inputs(d)
    o = W.alloc_outputs(d, fill_nan=False)
    tens = {n: to_device(x[n] if t["role"] == "in" else o[n], t["dtype"], "cuda")
            for n, t in d["tensors"].items() if t["role"] != "temp"}
    op.run(tens)
    op.run(tens)
    ops.append((name, op, tens, W.algorithmic_bytes(d)))
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
for name, op, tens, _ in ops:
    op.run(tens)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
for name, op, _, nb in ops:
    print(name, op.selected(0), nb)
