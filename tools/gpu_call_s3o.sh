python - > gpurun_out/trorder.log 2>&1 <<'PY'
import sys, os, json
sys.argv = ["x"]
sys.path.insert(0, "tools")
import importlib.util
spec = importlib.util.spec_from_file_location("tv", "tools/tr_variety.py"); m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m)
import torch, workloads as W
from bench import to_device
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp
cases = [("2-D f32 16384^2", lambda: W.transpose2d(16384, 16384, "f32")), ("2-D f16 8192x24576", lambda: W.transpose2d(8192, 24576, "f16")),
         ("cfg3", lambda: W.cfg3()), ("NHWC->NCHW", lambda: W.nhwc_to_nchw()), ("C=96", lambda: W.cfg3(256, 96, 56, 56))]
for name, mk in cases:
    d = mk()
    nbytes = W.algorithmic_bytes(d)
    x = W.make_inputs(d); o = W.alloc_outputs(d, fill_nan=False)
    copies = max(1, min(8, -(-3 * m.L2 // nbytes)))
    sets = [{n: to_device(x[n] if t["role"] == "in" else o[n], t["dtype"], "cuda") for n, t in d["tensors"].items() if t["role"] != "temp"} for _ in range(copies)]
    for var in ["0", "1", "2:4", "2:8", "2:16", "2:32"]:
        os.environ["FOP_TR_ORDER"] = var.split(":")[0]
        os.environ["FOP_TR_BV"] = var.split(":")[1] if ":" in var else "8"
        op = FusedOp(d, autotune=0)
        ms = m.time_op(lambda s: op.run(s), sets)
        print(json.dumps({"case": name, "order": var, "us": ms * 1e3, "GB_s": nbytes / ms / 1e6}), flush=True)
    del sets
    torch.cuda.empty_cache()
PY
echo rc=$?
cat gpurun_out/trorder.log | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); print(f\"{d['case']:22s} order {d['order']:5s} {d['us']:8.1f} us {d['GB_s']:7.0f} GB/s\")
    else: print(l.rstrip()[:200])
"
