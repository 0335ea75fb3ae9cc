"""fop_run_many: independent fused operators back to back on one stream, each
plan's first kernel launched with programmatic stream serialization (its
launch processed while the previous kernel runs; include/fop.h).  Results
must equal the plans run one by one (same plan objects, so the same tuned
kernels: bit for bit, reductions included), later work on the stream must
see every result (stream order kept), and the chain must be capturable in a
CUDA graph (bench.py replays one step as a graph)."""
import numpy as np
import pytest
import torch

import workloads as W
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, FopError, run_many


def _suite(small=True):
    if small:
        return [W.cfg2(4, 64, 28, 28), W.cfg3(8, 64, 14, 14), W.cfg4a(4, 64, 768), W.cfg4b(8192, 1024), W.cfg1()]
    return [W.cfg2(), W.cfg3(), W.cfg4a(), W.cfg4b()]


class _S:
    cuda_stream = 0


def test_run_many_rejects_peer_plans_before_launch(monkeypatch):
    op = FusedOp(W.cfg4b(256, 64), peer_world=2, peer_loop="r", jit=0)
    monkeypatch.setattr(op, "_check_tensor", lambda *a: None)   # host tensors stand in for device pointers
    t = {"x": torch.zeros(256 * 64, dtype=torch.float16), "out": torch.zeros(64)}
    with pytest.raises(FopError, match="fop_run_peer"):
        run_many([(op, t, torch.zeros(max(1, op.workspace_bytes), dtype=torch.uint8))], stream=_S())


def _outs(desc, dev):
    return {n: dev[n].clone() for n, t in desc["tensors"].items() if t["role"] in ("out", "inout")}


@pytest.mark.gpu
@pytest.mark.parametrize("small", [True, False])
def test_run_many_equals_one_by_one(small):
    from harness import device_tensors
    descs = _suite(small)
    ops = [FusedOp(d) for d in descs]
    devs = [device_tensors(d, W.make_inputs(d)) for d in descs]
    for op, dev in zip(ops, devs):      # tunes, then the reference results
        op.run(dev)
        op.run(dev)
    torch.cuda.synchronize()
    ref = [_outs(d, dev) for d, dev in zip(descs, devs)]
    for dev, d in zip(devs, descs):
        for n in _outs(d, dev):
            dev[n].fill_(float("nan"))
    run_many(list(zip(ops, devs)))
    got = [_outs(d, dev) for d, dev in zip(descs, devs)]   # clone() on the same stream: ordered after the chain
    torch.cuda.synchronize()
    for r, g in zip(ref, got):
        for n in r:
            assert torch.equal(r[n].view(torch.uint8), g[n].view(torch.uint8)), n


@pytest.mark.gpu
def test_run_many_completion_order():
    """A long kernel followed by a short one: work enqueued after the chain
    must not start before the LONG one has finished."""
    from harness import device_tensors
    big, tiny = W.cfg3(64, 256, 56, 56), W.cfg1()
    ops = [FusedOp(big), FusedOp(tiny)]
    devs = [device_tensors(big, W.make_inputs(big)), device_tensors(tiny, W.make_inputs(tiny))]
    ops[0].run(devs[0])
    torch.cuda.synchronize()
    want = devs[0]["out"].clone()
    for _ in range(5):
        devs[0]["out"].fill_(float("nan"))
        run_many(list(zip(ops, devs)))
        s = devs[0]["out"].clone()
        torch.cuda.synchronize()
        assert torch.equal(s.view(torch.int16), want.view(torch.int16))


@pytest.mark.gpu
def test_run_many_graph_capture():
    from harness import device_tensors
    descs = _suite(True)
    ops = [FusedOp(d) for d in descs]
    devs = [device_tensors(d, W.make_inputs(d)) for d in descs]
    for op, dev in zip(ops, devs):
        op.run(dev)
    torch.cuda.synchronize()
    ref = [_outs(d, dev) for d, dev in zip(descs, devs)]
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            run_many(list(zip(ops, devs)), stream=s)
    for dev, d in zip(devs, descs):
        for n in _outs(d, dev):
            dev[n].fill_(float("nan"))
    g.replay()
    torch.cuda.synchronize()
    for r, dev, d in zip(ref, devs, descs):
        for n in r:
            assert torch.equal(r[n].view(torch.uint8), dev[n].view(torch.uint8)), n
