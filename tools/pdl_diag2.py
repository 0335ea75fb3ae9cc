import sys
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import torch, workloads as W
from harness import device_tensors
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, run_many
d = W.cfg4b(8192, 1024)
import os; op = FusedOp(d, autotune=int(os.environ.get("AT", "1")))
dev = device_tensors(d, W.make_inputs(d))
op.run(dev); op.run(dev); torch.cuda.synchronize()
ref = dev["out"].clone()
print(op.selected(0), op.workspace_bytes, flush=True)
dev["out"].fill_(float("nan")); op.run(dev); torch.cuda.synchronize()
print("op.run nan:", int(torch.isnan(dev["out"]).sum()), flush=True)
dev["out"].fill_(float("nan")); run_many([(op, dev)]); torch.cuda.synchronize()
print("run_many nan:", int(torch.isnan(dev["out"]).sum()), flush=True)
dev["out"].fill_(float("nan")); op.run(dev); torch.cuda.synchronize()
print("op.run nan:", int(torch.isnan(dev["out"]).sum()), flush=True)
import os; print("emit", os.environ.get("FOP_PDL_EMIT"), "autotune", os.environ.get("AT"))

