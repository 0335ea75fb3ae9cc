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


def shard_desc(desc, loop, rank, world):
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
    info = {"partials": [], "slices": {}}
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
        if s.get("finalize"):
            raise ShardError(f"statement {i}: a finalize step cannot be applied to partial results")
        later_reads = [j for j in range(i + 1, len(desc["stmts"]))
                       if any(r[0] == s["write"][0] for r in desc["stmts"][j]["reads"])]
        if later_reads:
            raise ShardError(f"statement {i}: its partial result is consumed by statement {later_reads[0]}")
        info["partials"].append((s["write"][0], s.get("op", "sum")))
    return sh, info


def shard_inputs(desc, loop, rank, world, inputs):
    """Slice full host inputs (flat buffers of a contiguous layout) to the rank's block."""
    import numpy as np
    _, info = shard_desc(desc, loop, rank, world)
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


class ShardedFusedOp:
    """Plan the rank's sub-operator once; run = fop_run + all-reduce of partials."""

    def __init__(self, desc, loop, group=None, rank=None, world=None, **opts):
        from .fop import FusedOp
        self.group = group
        self.rank = dist.get_rank(group) if rank is None else rank
        self.world = dist.get_world_size(group) if world is None else world
        self.shard, self.info = shard_desc(desc, loop, self.rank, self.world)
        self.op = FusedOp(self.shard, **opts)

    def run(self, tensors, stream=None):
        self.op.run(tensors, stream=stream)
        if self.world > 1:
            allreduce_partials(tensors, self.info, self.group)
