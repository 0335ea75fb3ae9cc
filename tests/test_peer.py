"""Cross-GPU reductions fused into the COL_REDUCE kernel (fop.h peer groups;
SURVEY §8(e)): a reduction whose reduced loop is split across GPUs pushes its
partial sums into every rank's exchange buffer over NVLink peer memory and
adds all ranks' contributions in rank order inside the same kernel.

CPU tests: planner bookkeeping (which launch exchanges, buffer layout, what
is rejected), argument checks before any launch, the host-side handle
exchange over a world-size-2 gloo group, and a randomized-interleaving model
of the epoch/parity protocol.  GPU tests (one B200): W simulated ranks on W
streams of the same GPU — the kernels only see pointers, so the pushes, flags
and waits run exactly as across GPUs — checked against the oracle on the
WHOLE (unsharded) operator, bit-identical across ranks; repeated runs (epoch
and parity turnover); a peer that never arrives (bounded wait -> NaN + error
word); and two processes sharing one GPU through real CUDA IPC handles."""
import os
import random
import socket

import numpy as np
import pytest
import torch

import workloads as W
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, FopError
from paper_conf_cgo_bastoulzrlsjfjc22_b200.dist import shard_desc, shard_inputs, ShardError

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def colmean(R, C):
    d = W.cfg4b(R, C)
    d["name"] = "colmean"
    d["stmts"][0]["finalize"] = [("acc",), ("const", float(R)), ("div", 0, 1)]
    return d


def colmax(R, C):
    d = W.cfg4b(R, C)
    d["name"] = "colmax"
    d["stmts"][0]["op"] = "max"
    return d


# ---------------------------------------------------------------- CPU: planner
def test_peer_plan_layout():
    op = FusedOp(W.cfg4b(8192, 1024), peer_world=4, peer_loop="r", jit=0)
    L = op.info()["launches"]
    assert len(L) == 1 and L[0]["class"] == "col_reduce" and L[0]["peer_exchange"]
    # slab = 8 lanes x 8 f16 = 64 columns -> 16 slabs; [2][4][16][64] u64 | [16] u32 | error word
    al = lambda x: (x + 255) // 256 * 256  # noqa: E731
    assert op.peer_bytes == al(2 * 4 * 16 * 64 * 8) + al(16 * 4) + 16
    assert FusedOp(W.cfg4b(8192, 1024), jit=0).peer_bytes == 0


def test_peer_plan_has_no_tuning_variants():
    op = FusedOp(W.cfg4b(4096, 256), peer_world=2, peer_loop="r")
    assert op.selected(0)[0].endswith("_k0")
    src = op.source(0)
    assert "st_relaxed_sys_u64" in src and "wait_word" in src


def test_peer_parallel_loop_needs_no_exchange():
    # batch-parallel operators shard without communication: no exchange buffer
    assert FusedOp(W.cfg2(2, 8, 6, 16), peer_world=2, peer_loop="n", jit=0).peer_bytes == 0
    assert FusedOp(W.cfg4a(2, 6, 96), peer_world=2, peer_loop="b", jit=0).peer_bytes == 0


def test_peer_rejections():
    with pytest.raises(FopError) as e:        # row reduction over the split loop (vector loop = reduced loop)
        FusedOp(W.cfg4a(2, 6, 96), peer_world=2, peer_loop="h", jit=0)
    assert e.value.status == "FOP_E_UNSUPPORTED"
    d = W.cfg4b(64, 32)                        # a later statement consumes the partial sum
    d["tensors"]["y"] = {"shape": [64, 32], "dtype": "f32", "role": "out"}
    d["stmts"].append({"kind": "assign", "loops": ["r", "c"], "write": ("y", ["r", "c"]),
                       "reads": [("x", ["r", "c"]), ("out", ["c"])], "expr": [("load", 0), ("load", 1), ("div", 0, 1)]})
    with pytest.raises(FopError) as e:
        FusedOp(d, peer_world=2, peer_loop="r", jit=0)
    assert e.value.status == "FOP_E_UNSUPPORTED"
    for bad in (dict(peer_world=9, peer_loop="r"), dict(peer_world=-1, peer_loop="r"),
                dict(peer_world=2, peer_loop=7)):
        with pytest.raises(FopError) as e:
            FusedOp(W.cfg4b(64, 32), jit=0, **bad)
        assert e.value.status == "FOP_E_INVALID"


class _S:
    cuda_stream = 0


def test_peer_run_argument_checks_before_launch(monkeypatch):
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import PeerGroup
    op = FusedOp(W.cfg4b(256, 64), peer_world=2, peer_loop="r", jit=0)
    # host tensors stand in for device pointers: these are the C library's own
    # checks (before any launch), so the binding's device check is bypassed
    monkeypatch.setattr(op, "_check_tensor", lambda *a: None)
    monkeypatch.setattr(op, "_check_workspace", lambda *a: None)
    t = {"x": torch.zeros(256 * 64, dtype=torch.float16), "out": torch.zeros(64)}
    ws = torch.zeros(max(1, op.workspace_bytes), dtype=torch.uint8)
    with pytest.raises(FopError, match="fop_run_peer"):
        op.run(t, workspace=ws, stream=_S())
    with pytest.raises(FopError, match="world"):
        op.run(t, workspace=ws, stream=_S(), peers=PeerGroup(0, [4096, 8192, 12288]))
    with pytest.raises(FopError, match="aligned"):
        op.run(t, workspace=ws, stream=_S(), peers=PeerGroup(0, [4096, 8200]))


def test_shard_desc_fused_allows_finalize():
    d = colmean(512, 40)
    with pytest.raises(ShardError):
        shard_desc(d, "r", 0, 2)
    sh, info = shard_desc(d, "r", 1, 2, fused=True)
    assert info["partials"] == [("out", "sum")] and sh["loops"]["r"] == 256


# ---------------------------------------------------------------- CPU: protocol model
def _simulate(world, runs, seed):
    """Random interleaving of the kernel epilogue's steps on `world` ranks
    (each rank's runs in stream order).  Every word carries (value, epoch)
    atomically; a receiver polls each word until its epoch is the run's.
    Checks that every accepted word is that sender's value of the same run."""
    rng = random.Random(seed)
    words = [[[(None, 0)] * world for _ in range(2)] for _ in range(world)]   # [recv][parity][sender]
    ctr = [0] * world

    def rank_prog(r):
        for run in range(runs):
            ep = ctr[r] + 1
            ctr[r] = ep
            assert ep == run + 1
            for q in rng.sample(range(world), world):       # stores land in any order
                words[q][ep & 1][r] = ((r, ep), ep)
                yield
            for q in rng.sample(range(world), world):       # polls in any order
                while words[r][ep & 1][q][1] != ep:
                    yield
                assert words[r][ep & 1][q][0] == (q, ep), (r, q, ep, words[r][ep & 1][q])
                yield
    progs = {r: rank_prog(r) for r in range(world)}
    while progs:
        r = rng.choice(list(progs))
        try:
            next(progs[r])
        except StopIteration:
            del progs[r]


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_exchange_protocol_model(world):
    for seed in range(40):
        _simulate(world, runs=6, seed=seed)


# ---------------------------------------------------------------- CPU: handle exchange (gloo, 2 ranks)
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _px_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    import torch.distributed as dist
    from paper_conf_cgo_bastoulzrlsjfjc22_b200.dist import PeerExchange
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        fake = {"alloc": lambda n: (0x10000 * (rank + 1), bytes([rank + 1]) * 64),
                "open": lambda h: 0x7f0000 + h[0]}
        px = PeerExchange(512, rank=rank, world=world, _alloc=fake["alloc"], _open=fake["open"])
        q.put((rank, px.bufs, px.peers.rank, px.peers.world))
        px.close(_close=lambda p: None, _free=lambda p: None)
    finally:
        dist.destroy_process_group()


def test_peer_exchange_handles_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_px_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    # rank 0: own buffer, then rank 1's handle opened; rank 1: rank 0's opened, then own
    assert res[0] == (0, [0x10000, 0x7f0000 + 2], 0, 2)
    assert res[1] == (1, [0x7f0000 + 1, 0x20000], 1, 2)


# ---------------------------------------------------------------- GPU
def _simulated_group(desc, loop, world, opts=None, runs=1, seeds=None):
    """Run the sharded operator as `world` ranks on one GPU: one stream, one
    workspace, one exchange buffer per rank; every rank's launch enqueued
    before any is waited on.  Returns per run: (inputs of the whole operator,
    [rank outputs])."""
    from harness import device_tensors, to_host
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import PeerGroup
    sh, info = shard_desc(desc, loop, 0, world, fused=True)
    op = FusedOp(sh, peer_world=world, peer_loop=loop, **(opts or {}))
    assert op.info()["launches"][-1]["peer_exchange"]
    bufs = [torch.zeros(op.peer_bytes, dtype=torch.uint8, device="cuda") for _ in range(world)]
    ptrs = [b.data_ptr() for b in bufs]
    wss = [torch.zeros(max(1, op.workspace_bytes), dtype=torch.uint8, device="cuda") for _ in range(world)]
    streams = [torch.cuda.Stream() for _ in range(world)]
    out = []
    for k in range(runs):
        x = W.make_inputs(desc, seed_offset=(seeds[k] if seeds else 100 * k))
        devs = [device_tensors(sh, shard_inputs(desc, loop, r, world, x)) for r in range(world)]
        torch.cuda.synchronize()
        for r in range(world):
            op.run(devs[r], workspace=wss[r], stream=streams[r], peers=PeerGroup(r, ptrs))
        torch.cuda.synchronize()
        res = [{n: to_host(devs[r][n], sh["tensors"][n]["dtype"]) for n, _ in info["partials"]}
               for r in range(world)]
        out.append((x, res))
    errs = [int(b[-16:].view(torch.int32)[0]) for b in bufs]
    return out, errs


def _check_combined(desc, x, res, tol):
    from oracle import oracle as O
    from harness import abs_terms_desc, assert_normwise
    ref = O.run(desc, x)
    scale = O.run(abs_terms_desc(desc, 0), x)
    for r in range(1, len(res)):
        assert np.array_equal(res[r]["out"].view(np.uint32), res[0]["out"].view(np.uint32)), f"rank {r} differs"
    if desc["stmts"][0].get("op") == "max":
        assert np.array_equal(res[0]["out"], ref["out"])     # max is exact in any order
    else:
        assert_normwise(res[0]["out"], ref["out"], scale["out"], tol, "out")


@pytest.mark.gpu
@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_peer_colsum_simulated_ranks(world):
    desc = W.cfg4b(2048 * world, 1024)
    out, errs = _simulated_group(desc, "r", world, runs=3)
    assert errs == [0] * world
    for x, res in out:
        _check_combined(desc, x, res, 1e-5)


@pytest.mark.gpu
@pytest.mark.parametrize("make,R,C,world", [(colmean, 3000, 1000, 2), (colmax, 1024, 136, 4),
                                            (W.cfg4b, 64, 8, 8), (W.cfg4b, 24, 4096, 3)])
def test_peer_ragged_finalize_max(make, R, C, world):
    desc = make(R * world, C)
    out, errs = _simulated_group(desc, "r", world, runs=2)
    assert errs == [0] * world
    for x, res in out:
        _check_combined(desc, x, res, 1e-5)


@pytest.mark.gpu
def test_peer_many_runs_epoch_turnover():
    desc = W.cfg4b(4 * 512, 256)
    out, errs = _simulated_group(desc, "r", 4, runs=9)
    assert errs == [0] * 4
    for x, res in out:
        _check_combined(desc, x, res, 1e-5)


@pytest.mark.gpu
def test_peer_absent_rank_times_out():
    from harness import device_tensors, to_host
    from paper_conf_cgo_bastoulzrlsjfjc22_b200 import PeerGroup
    desc = W.cfg4b(1024, 128)
    sh, _ = shard_desc(desc, "r", 0, 2, fused=True)
    op = FusedOp(sh, peer_world=2, peer_loop="r", peer_timeout_ms=50)
    bufs = [torch.zeros(op.peer_bytes, dtype=torch.uint8, device="cuda") for _ in range(2)]
    dev = device_tensors(sh, shard_inputs(desc, "r", 0, 2, W.make_inputs(desc)))
    op.run(dev, peers=PeerGroup(0, [b.data_ptr() for b in bufs]))    # rank 1 never runs
    torch.cuda.synchronize()
    assert np.isnan(to_host(dev["out"], "f32")).all()
    assert int(bufs[0][-16:].view(torch.int32)[0]) == 1


def _ipc_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch.distributed as dist
    from harness import device_tensors, to_host
    from paper_conf_cgo_bastoulzrlsjfjc22_b200.dist import ShardedFusedOp
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    torch.zeros(1, device="cuda")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        desc = W.cfg4b(2 * 4096, 512)
        sop = ShardedFusedOp(desc, "r", rank=rank, world=world, exchange="peer")
        outs = []
        for k in range(3):
            x = W.make_inputs(desc, seed_offset=7 * k)
            dev = device_tensors(sop.shard, shard_inputs(desc, "r", rank, world, x))
            sop.run(dev)
            torch.cuda.synchronize()
            outs.append(to_host(dev["out"], "f32"))
        sop.close()
        q.put((rank, outs))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.timeout(300)
def test_peer_ipc_two_processes_one_gpu():
    """Real CUDA IPC handles (fop_peer_alloc / fop_peer_open) between two
    processes on the same GPU; the device-side wait spans the two contexts."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=240) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    desc = W.cfg4b(2 * 4096, 512)
    for k in range(3):
        x = W.make_inputs(desc, seed_offset=7 * k)
        _check_combined(desc, x, [{"out": res[0][1][k]}, {"out": res[1][1][k]}], 1e-5)
