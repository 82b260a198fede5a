"""Multi-GPU root sharding (one process per GPU, torch.distributed plumbing).

North star: "Work is partitioned ... by sharding first-level root vertices,
whose subtrees are independent, with a small NCCL max-allreduce of the omega
lower bound each level and a final gather of the cliques over NVLink."

 * every rank loads the whole graph; rank 0 runs the k-core peel and
   broadcasts its core numbers and peel order (one int32[2n] broadcast over
   NVLink), the other ranks install them with mce_set_core instead of peeling,
   and every rank orients its edges from them -- identically, which clique
   ownership depends on (the asynchronous peel's order depends on timing).
   orientation="degeneracy_det" instead has every rank compute the
   deterministic order (core, shell round, id) itself, with no broadcast but
   a slower peel (reading 18); the degree orientation is a function
   of the graph and needs neither;
 * heuristic seeds are dealt cyclically (seed position % world == rank) and
   root vertices by CSR id (id % world == rank) inside the library
   (mce_options.shard_rank / shard_count), or level-d candidates by path hash
   (shard_depth d >= 2);
 * after every expansion step the library calls `bound_sync`, which
   max-allreduces (best clique size, still-active flag) across ranks, so a
   clique found on one GPU tightens the pruning bound on all of them and the
   ranks stay in lock-step until the last one finishes;
 * the ranks whose best equals the global omega contribute their cliques to
   one all-gather (multiplicities add: root subtrees are disjoint).
"""

from __future__ import annotations

import os
from typing import Optional

import numpy as np
import torch
import torch.distributed as dist

from .api import Graph, Result


def _device(group) -> torch.device:
    if dist.get_backend(group) == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def make_bound_sync(group=None):
    """The per-step exchange: (local best, local active) -> (global best, any active)."""
    dev = _device(group)

    def sync(local_best: int, local_active: int):
        t = torch.tensor([local_best, local_active], dtype=torch.int64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        v = t.tolist()
        return int(v[0]), int(v[1])

    return sync


def gather_result(res: Result, group=None, find_one: bool = False, max_cliques: int = 0) -> Result:
    """Combine per-rank results: global omega, summed multiplicity, all cliques."""
    dev = _device(group)
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if os.environ.get("MCE_DEBUG_GATHER"):
        print(f"[gather] rank {rank}/{world}: local omega {res.omega} count {res.count} "
              f"stored {res.cliques.shape[0]}", flush=True)
    t = torch.tensor([res.omega], dtype=torch.int64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    omega = int(t.item())
    mine = res.cliques if res.omega == omega else np.zeros((0, omega), np.int32)
    count = res.count if res.omega == omega else 0
    if find_one:  # the lowest rank holding a clique of size omega provides it
        holder = torch.tensor([rank if res.omega == omega else world], dtype=torch.int64, device=dev)
        dist.all_reduce(holder, op=dist.ReduceOp.MIN, group=group)
        src = int(holder.item())
        buf = torch.zeros(max(omega, 1), dtype=torch.int64, device=dev)
        if rank == src and omega > 0:
            buf[:omega] = torch.from_numpy(mine[0].astype(np.int64)).to(dev)
        dist.broadcast(buf, src=dist.get_global_rank(group, src) if group is not None else src, group=group)
        cl = buf[:omega].cpu().numpy().astype(np.int32).reshape(1, omega)
        return Result(omega, 1, cl, False, res.levels, res.timing)
    # only ranks holding cliques of the global omega count (their lists are the ones kept)
    c = torch.tensor([count, int(res.truncated) if res.omega == omega else 0], dtype=torch.int64, device=dev)
    dist.all_reduce(c, op=dist.ReduceOp.SUM, group=group)
    total, trunc = (int(x) for x in c.tolist())
    n_local = torch.tensor([mine.shape[0]], dtype=torch.int64, device=dev)
    sizes = [torch.zeros_like(n_local) for _ in range(world)]
    dist.all_gather(sizes, n_local, group=group)
    sizes = [int(s.item()) for s in sizes]
    mx = max(sizes) if sizes else 0
    width = max(omega, 1)
    pad = torch.zeros((max(mx, 1), width), dtype=torch.int64, device=dev)
    if mine.shape[0] and omega > 0:
        pad[: mine.shape[0], :omega] = torch.from_numpy(mine.astype(np.int64)).to(dev)
    parts = [torch.zeros_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad, group=group)
    rows = [p[:s, :omega].cpu().numpy() for p, s in zip(parts, sizes)]
    allrows = np.concatenate(rows, 0).astype(np.int32) if rows else np.zeros((0, omega), np.int32)
    if allrows.shape[0] > 1 and omega > 0:
        allrows = allrows[np.lexsort(allrows.T[::-1])]
    if max_cliques > 0 and allrows.shape[0] > max_cliques:  # each rank stored up to max_cliques
        allrows = allrows[:max_cliques]
        trunc = 1
    return Result(omega, total, allrows, bool(trunc), res.levels, res.timing)


def agree_core(graph: Graph, group=None):
    """Rank 0 peels (or reuses its cached peel) and broadcasts its core numbers
    and degeneracy order; the others set them (mce_set_core) so every rank
    orients the edges identically with one peel in the whole job."""
    if dist.get_world_size(group) == 1 or graph.n == 0:
        return
    n = graph.n
    dev = torch.device("cuda", graph.device) if _device(group).type == "cuda" else torch.device("cpu")
    buf = torch.empty(2 * n, dtype=torch.int32, device=dev)
    src = dist.get_global_rank(group, 0) if group is not None else 0
    if dist.get_rank(group) == 0:
        graph.core_into(buf[:n], buf[n:])
    dist.broadcast(buf, src=src, group=group)
    if dist.get_rank(group) != 0:
        graph.set_core(buf[:n], buf[n:])


def _agree(graph: Graph, group, world: int, opts: dict):
    if world > 1 and opts.setdefault("orientation", "degeneracy") == "degeneracy":
        agree_core(graph, group)


def agree_orientation(graph: Graph, group=None, orientation: str = "degeneracy"):
    """Fallback for callers that need rank 0's own (asynchronous-peel) order on
    every rank: broadcast it and set it on the others (each rank re-peels for
    its core numbers; enumerate_distributed / find_one_distributed use
    agree_core, which broadcasts those too)."""
    if dist.get_world_size(group) == 1 or graph.n == 0:
        return
    dev = _device(group)
    if dev.type == "cuda":
        order = torch.empty(graph.n, dtype=torch.int32, device=torch.device("cuda", graph.device))
    else:
        order = torch.empty(graph.n, dtype=torch.int32)
    src = dist.get_global_rank(group, 0) if group is not None else 0
    if dist.get_rank(group) == 0:
        graph.order_into(order, orientation)
    dist.broadcast(order, src=src, group=group)
    if dist.get_rank(group) != 0:
        graph.set_order(order, orientation)


def enumerate_distributed(graph: Graph, group=None, **opts) -> Result:
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    _agree(graph, group, world, opts)
    res = graph.enumerate(shard_rank=rank, shard_count=world, bound_sync=make_bound_sync(group), **opts)
    return gather_result(res, group, max_cliques=int(opts.get("max_cliques", 0) or 0))


def find_one_distributed(graph: Graph, window: int = 0, group=None, **opts) -> Result:
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    _agree(graph, group, world, opts)
    res = graph.find_one(window=window, shard_rank=rank, shard_count=world, bound_sync=make_bound_sync(group),
                         **opts)
    return gather_result(res, group, find_one=True)


def shard_of(index: int, world: int) -> int:
    """Rank that owns root (or heuristic seed) number `index` of the sorted list."""
    return index % world


def owned(count: int, rank: int, world: int, offset: Optional[int] = None) -> range:
    """Items 0..count-1 owned by `rank` under the cyclic deal the library uses for seeds and root ids."""
    return range(rank if offset is None else offset, count, world)
