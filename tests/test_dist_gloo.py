"""Multi-process (world_size 2, gloo, CPU) tests of the batch-sharding logic
(paper_conf_cgo_bastoulzrlsjfjc22_b200.dist).  Each rank evaluates its shard
with the oracle standing in for its GPU, partial reductions are all-reduced
over gloo exactly as bench.py does over NCCL, and the gathered result must
equal the oracle on the whole operator: bitwise for batch-parallel operators,
within the R16 normwise bound for the sharded column sum."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import workloads as W
from paper_conf_cgo_bastoulzrlsjfjc22_b200.dist import ShardError, shard_desc, shard_inputs, allreduce_partials


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


CASES = {
    "cfg2": (lambda: W.cfg2(4, 8, 6, 10), "n"),
    "cfg3": (lambda: W.cfg3(4, 16, 5, 6), "n"),
    "cfg4a": (lambda: W.cfg4a(4, 6, 96), "b"),
    "cfg4b": (lambda: W.cfg4b(512, 40), "r"),
}


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        from oracle import oracle as O
        mk, loop = CASES[case]
        d = mk()
        x = W.make_inputs(d)
        sh, info = shard_desc(d, loop, rank, world)
        xs = shard_inputs(d, loop, rank, world, x)
        res = O.run(sh, xs)
        tens = {n: torch.from_numpy(v.astype(np.float32) if v.dtype == np.float32 else v.copy())
                for n, v in res.items()}
        allreduce_partials(tens, info)
        # gather every output to rank 0
        out = {}
        for n, t in tens.items():
            if d["tensors"][n]["role"] != "out":
                continue
            ts = t.contiguous().view(torch.uint8)          # gloo: gather raw bytes
            parts = [torch.empty_like(ts) for _ in range(world)]
            dist.all_gather(parts, ts)
            out[n] = [p.numpy().view(res[n].dtype) for p in parts]
        q.put((rank, out, info))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", list(CASES))
def test_sharded_equals_whole(case):
    from oracle import oracle as O
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in ps:
        p.start()
    results = [q.get(timeout=120) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    rank0 = [r for r in results if r[0] == 0][0]
    out, info = rank0[1], rank0[2]
    mk, loop = CASES[case]
    d = mk()
    x = W.make_inputs(d)
    ref = O.run(d, x)
    for n, parts in out.items():
        t = d["tensors"][n]
        if n in info["slices"]:
            dim = info["slices"][n][0]
            shp = list(t["shape"])
            shp[dim] //= world
            full = np.concatenate([p.reshape(shp) for p in parts], axis=dim).reshape(-1)
            assert np.array_equal(full.view(np.uint8), ref[n].view(np.uint8)), n
        else:   # all-reduced partial: every rank holds the same full result
            assert np.array_equal(parts[0], parts[1])
            scale = np.abs(x["x"].astype(np.float64)).reshape(-1, 40).sum(0)
            err = np.abs(parts[0].astype(np.float64) - ref[n].astype(np.float64))
            assert np.all(err <= 1e-5 * scale + 1e-30), n


def test_shard_desc_rules():
    d = W.cfg4b(512, 40)
    sh, info = shard_desc(d, "r", 1, 4)
    assert sh["loops"]["r"] == 128 and info["partials"] == [("out", "sum")]
    assert sh["tensors"]["x"]["shape"] == [128, 40] and info["slices"]["x"] == (0, 128, 256)
    d = W.cfg4a(4, 6, 96)
    with pytest.raises(ShardError):          # mean's finalize (/H) on partial sums
        shard_desc(d, "h", 0, 2)
    sh, info = shard_desc(d, "b", 0, 2)
    assert info["partials"] == [] and sh["tensors"]["mean"]["shape"] == [2, 6]
    with pytest.raises(ShardError):
        shard_desc(W.cfg2(3, 8, 6, 10), "n", 0, 2)   # 3 not divisible by 2


@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_strong_scaling_shards_tile_cfg5(world):
    """bench.py --scaling strong: BASELINE.json's cfg5 (4x the batch of configs[1..3]) split over
    N ranks — the shards' batch blocks are disjoint, cover the global operator, carry equal
    algorithmic bytes, and only cfg4b (rows = its reduced axis) produces partials."""
    import bench
    for name, (gmk, loop) in bench.GLOBAL.items():
        g = gmk(bench.STRONG_SCALE)
        E = g["loops"][loop]
        blocks, nbytes = [], set()
        for r in range(world):
            sh, info = shard_desc(g, loop, r, world, fused=True)
            assert sh["loops"][loop] == E // world
            blocks += [info["slices"][n][1:] for n in info["slices"]][:1]
            nbytes.add(W.algorithmic_bytes(sh))
            assert [p[0] for p in info["partials"]] == (["out"] if name == "cfg4b" else [])
        assert sorted(blocks) == [(r * E // world, (r + 1) * E // world) for r in range(world)]
        assert len(nbytes) == 1
        if world == 1:
            assert nbytes.pop() == W.algorithmic_bytes(g)
