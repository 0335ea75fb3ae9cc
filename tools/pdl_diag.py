import sys, os
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import torch, workloads as W
from harness import device_tensors
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, run_many
def outs(d, dev): return {n: dev[n] for n, t in d["tensors"].items() if t["role"] in ("out","inout")}
combos = [["cfg4a","cfg4b"], ["cfg4b","cfg1"], ["cfg2","cfg4b"], ["cfg4b","cfg4b2"], ["cfg3","cfg4a","cfg4b","cfg1"]]
mk = {"cfg1": W.cfg1, "cfg2": lambda: W.cfg2(4,64,28,28), "cfg3": lambda: W.cfg3(8,64,14,14), "cfg4a": lambda: W.cfg4a(4,64,768), "cfg4b": lambda: W.cfg4b(8192,1024), "cfg4b2": lambda: W.cfg4b(4096,512)}
for combo in combos:
    descs = [mk[c]() for c in combo]
    ops = [FusedOp(d) for d in descs]
    devs = [device_tensors(d, W.make_inputs(d)) for d in descs]
    for op, dev in zip(ops, devs): op.run(dev); op.run(dev)
    torch.cuda.synchronize()
    ref = [{n: v.clone() for n, v in outs(d, dev).items()} for d, dev in zip(descs, devs)]
    for mode in ["sync", "nosync"]:
        for d, dev in zip(descs, devs):
            for v in outs(d, dev).values(): v.fill_(float("nan"))
        run_many(list(zip(ops, devs)))
        if mode == "sync": torch.cuda.synchronize()
        got = [{n: v.clone() for n, v in outs(d, dev).items()} for d, dev in zip(descs, devs)]
        torch.cuda.synchronize()
        bad = [(c, n, int(torch.isnan(got[i][n].float()).sum()), bool(torch.equal(got[i][n].view(torch.uint8), ref[i][n].view(torch.uint8)))) for i, c in enumerate(combo) for n in ref[i]]
        print(combo, mode, bad, flush=True)
