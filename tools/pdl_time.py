"""Time the bench suite chain (cfg2, cfg3, cfg4a, cfg4b) per step: fop_run per
op vs fop_run_many, eager and inside a CUDA graph (no host overhead)."""
import sys, os, json
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import torch, workloads as W
from harness import device_tensors
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, run_many
descs = [W.cfg2(), W.cfg3(), W.cfg4a(), W.cfg4b()]
ops = [FusedOp(d) for d in descs]
devs = [device_tensors(d, W.make_inputs(d)) for d in descs]
for op, dev in zip(ops, devs):
    op.run(dev); op.run(dev)
torch.cuda.synchronize()
items = list(zip(ops, devs))
def one_by_one():
    for op, dev in items: op.run(dev)
def many():
    run_many(items)
def t(fn, reps=50):
    for _ in range(5): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps * 1e3
res = {"eager_one_by_one_us": t(one_by_one), "eager_run_many_us": t(many)}
import time
t0 = time.perf_counter()
for _ in range(100): many()
res["host_run_many_us"] = (time.perf_counter() - t0) / 100 * 1e6
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(100): one_by_one()
res["host_one_by_one_us"] = (time.perf_counter() - t0) / 100 * 1e6
torch.cuda.synchronize()
for name, fn in (("graph_one_by_one_us", one_by_one), ("graph_run_many_us", many)):
    g = torch.cuda.CUDAGraph(); st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        with torch.cuda.graph(g, stream=st):
            for _ in range(10): fn()
    res[name] = t(lambda: g.replay(), reps=10) / 10
print(json.dumps({k: round(v, 1) for k, v in res.items()}), flush=True)
