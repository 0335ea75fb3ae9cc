"""Multi-GPU partitioning of fused operators (BASELINE.json
north_star (4)): one process per GPU, the fused operator split along its
outermost parallel (batch) loop, NCCL over NVLink only where a reduction's
reduced axis is the sharded one.

The paper itself is single-GPU; the split follows from the
operator's semantics: iterations of a loop that indexes every written tensor
(a parallel loop) are independent, so contiguous blocks of it go to ranks
with no communication.  If the loop is a REDUCTION loop of some statement
(its target does not use the loop) each rank produces a partial result and
one all-reduce (SUM or MAX) combines them — that is legal only when nothing
after the reduction consumes it inside the operator and the statement has no
finalize step (finalize(a+b) != finalize(a)+finalize(b) in general).

    sh = shard_desc(desc, "r", rank, world)       # the rank's sub-operator
    op = ShardedFusedOp(desc, "r", group=pg)      # plan + run + all-reduce

Two ways to combine partial results:
  exchange="peer" (default on GPUs): the reduction kernel itself pushes its
      partial sums into every rank's exchange buffer over NVLink peer memory
      and adds all ranks' contributions in rank order (fop_run_peer; one
      kernel per rank, no separate collective; identical bits on all ranks;
      a finalize step is then legal because it runs after the combine);
  exchange="nccl": fop_run, then one NCCL all-reduce per partial tensor.
"""
import copy

import torch
import torch.distributed as dist


class ShardError(ValueError):
    pass


def _index_loops(index):
    out = []
    for e in index:
        if isinstance(e, str):
            out.append(e)
        elif isinstance(e, (tuple, list)):
            out.append(e[0])
        else:
            out.append(None)
    return out


def shard_desc(desc, loop, rank, world, fused=False):
    """Sub-operator of `rank` when `loop` is split in `world` contiguous blocks.

    Returns (shard, info): `shard` is a description whose tensors are the
    rank-local blocks (contiguous, ready to allocate on the rank's GPU);
    info = {"partials": [(tensor, "sum"|"max")], "slices": {tensor: (dim, start, stop)}}
    """
    E = desc["loops"][loop]
    if E % world:
        raise ShardError(f"extent {E} of loop {loop!r} is not divisible by {world}")
    blk = E // world
    sh = copy.deepcopy(desc)
    sh["loops"][loop] = blk
    info = {"partials": [], "slices": {}, "loop": loop}
    # every tensor dim indexed by `loop` is cut to the rank's block
    dims = {}
    for s in desc["stmts"]:
        for name, index in [s["write"]] + list(s["reads"]):
            for d, l in enumerate(_index_loops(index)):
                if l == loop:
                    if isinstance(index[d], (tuple, list)) and index[d][1] != 0:
                        raise ShardError(f"{name}: offset access along the sharded loop")
                    if dims.get(name, d) != d:
                        raise ShardError(f"{name}: sharded loop indexes two dims")
                    dims[name] = d
    for name, d in dims.items():
        t = sh["tensors"][name]
        if t.get("strides"):
            raise ShardError(f"{name}: explicit strides are not sharded (allocate contiguous shards)")
        if t["shape"][d] != E:
            raise ShardError(f"{name}: dim {d} has extent {t['shape'][d]} != loop extent {E}")
        t["shape"] = list(t["shape"])
        t["shape"][d] = blk
        info["slices"][name] = (d, rank * blk, (rank + 1) * blk)
    # statements reducing over the sharded loop produce partials
    for i, s in enumerate(desc["stmts"]):
        if loop not in s["loops"]:
            continue
        wl = _index_loops(s["write"][1])
        if loop in wl:
            continue
        if s["kind"] != "reduce":
            raise ShardError(f"statement {i} writes {s['write'][0]} repeatedly along {loop!r}")
        if s.get("finalize") and not fused:
            raise ShardError(f"statement {i}: a finalize step cannot be applied to partial results "
                             "(use the fused peer exchange, which finalizes after the combine)")
        later_reads = [j for j in range(i + 1, len(desc["stmts"]))
                       if any(r[0] == s["write"][0] for r in desc["stmts"][j]["reads"])]
        if later_reads:
            raise ShardError(f"statement {i}: its partial result is consumed by statement {later_reads[0]}")
        info["partials"].append((s["write"][0], s.get("op", "sum")))
    return sh, info


def shard_inputs(desc, loop, rank, world, inputs):
    """Slice full host inputs (flat buffers of a contiguous layout) to the rank's block."""
    import numpy as np
    _, info = shard_desc(desc, loop, rank, world, fused=True)   # slices only
    out = {}
    for name, buf in inputs.items():
        if name not in info["slices"]:
            out[name] = buf
            continue
        d, a, b = info["slices"][name]
        shape = desc["tensors"][name]["shape"]
        out[name] = np.ascontiguousarray(buf.reshape(shape).take(range(a, b), axis=d)).reshape(-1)
    return out


_RED = {"sum": dist.ReduceOp.SUM, "max": dist.ReduceOp.MAX}


def allreduce_partials(tensors, info, group=None):
    """Combine the partial results of reductions over the sharded loop
    (one all-reduce per partial tensor; NCCL over NVLink on GPU ranks)."""
    for name, op in info["partials"]:
        dist.all_reduce(tensors[name], op=_RED[op], group=group)


class PeerExchange:
    """The exchange buffers of one peer-exchanging plan across a process group
    (fop.h, peer groups): each rank allocates its zero-filled buffer with
    fop_peer_alloc, the 64-byte CUDA IPC handles are all-gathered over the
    process group, and every other rank's buffer is mapped with fop_peer_open
    (NVLink peer access).  `self.peers` is the fop_peer_group to run with."""

    def __init__(self, nbytes, group=None, rank=None, world=None, _alloc=None, _open=None):
        from . import fop as F
        alloc = _alloc or F.peer_alloc
        open_ = _open or F.peer_open
        self.rank = dist.get_rank(group) if rank is None else rank
        self.world = dist.get_world_size(group) if world is None else world
        self.nbytes = nbytes
        self.local, handle = alloc(nbytes)
        handles = [None] * self.world
        dist.all_gather_object(handles, (self.rank, nbytes, handle), group=group)
        for q, (r, n, _) in enumerate(handles):
            if r != q or n != nbytes:
                raise ShardError(f"rank {q}: exchange buffer of {n} bytes (rank {r}) does not match {nbytes}")
        self.opened = {q: open_(handles[q][2]) for q in range(self.world) if q != self.rank}
        self.bufs = [self.local if q == self.rank else self.opened[q] for q in range(self.world)]
        self.peers = F.PeerGroup(self.rank, self.bufs)

    def close(self, _close=None, _free=None):
        from . import fop as F
        for p in self.opened.values():
            (_close or F.peer_close)(p)
        (_free or F.peer_free)(self.local)
        self.opened, self.local = {}, None


class ShardedFusedOp:
    """Plan the rank's sub-operator once; run = the rank's kernels with the
    partial results combined in the reduction kernel over NVLink
    (exchange="peer") or fop_run + an NCCL all-reduce (exchange="nccl")."""

    def __init__(self, desc, loop, group=None, rank=None, world=None, exchange="peer", **opts):
        from .fop import FusedOp
        self.group = group
        self.rank = dist.get_rank(group) if rank is None else rank
        self.world = dist.get_world_size(group) if world is None else world
        self.exchange = exchange
        fused = exchange == "peer"
        self.shard, self.info = shard_desc(desc, loop, self.rank, self.world, fused=fused)
        if fused and self.info["partials"]:
            opts = dict(opts, peer_world=self.world, peer_loop=loop)
        self.op = FusedOp(self.shard, **opts)
        self.px = PeerExchange(self.op.peer_bytes, group, self.rank, self.world) if self.op.peer_bytes else None

    def run(self, tensors, stream=None):
        if self.px is not None:
            self.op.run(tensors, stream=stream, peers=self.px.peers)
            return
        self.op.run(tensors, stream=stream)
        if self.world > 1:
            allreduce_partials(tensors, self.info, self.group)

    def close(self):
        if self.px is not None:
            import torch as _t
            _t.cuda.synchronize()
            self.px.close()
            self.px = None
