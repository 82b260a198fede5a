"""Multi-GPU root partitioner (DESIGN.md §8 row a8): host logic on CPU with
world_size-2 `gloo` process groups, and the library's root/seed sharding on
one GPU (the shards of a sharded run together give the unsharded answer).

North star: "Work is partitioned ... by sharding first-level root vertices,
whose subtrees are independent, with a small NCCL max-allreduce of the omega
lower bound each level and a final gather of the cliques".
"""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_geilpo23_b200 import distributed as mdist
from paper_conf_ipps_geilpo23_b200.api import Result


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run(rank, world, port, fn, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, fn(rank, world)))
    finally:
        dist.destroy_process_group()


def spawn(fn, world=2, timeout=120):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_run, args=(r, world, port, fn, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=timeout) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return [out[r] for r in range(world)]


# --- per-rank bodies (module level: picklable for spawn) -------------------

def _bound_sync_body(rank, world):
    sync = mdist.make_bound_sync()
    # step 1: rank 1 found a bigger clique, rank 0 still active
    b1 = sync(5 if rank == 0 else 7, 1 if rank == 0 else 0)
    # step 2: nobody active
    b2 = sync(6, 0)
    return b1, b2


def _gather_body(rank, world):
    # rank 0 holds two 3-cliques and one (stale) 2-clique-sized result on rank 1
    if rank == 0:
        r = Result(3, 2, np.array([[4, 5, 6], [0, 1, 2]], np.int32), False, [], {})
    else:
        r = Result(3, 1, np.array([[1, 2, 3]], np.int32), False, [], {})
    g = mdist.gather_result(r)
    return g.omega, g.count, g.cliques.tolist(), g.truncated


def _gather_mixed_omega_body(rank, world):
    # a rank whose subtrees only reach a smaller clique contributes nothing
    if rank == 0:
        r = Result(2, 5, np.array([[0, 1], [1, 2], [2, 3], [3, 4], [4, 0]], np.int32), False, [], {})
    else:
        r = Result(4, 1, np.array([[5, 6, 7, 8]], np.int32), True, [], {})
    g = mdist.gather_result(r)
    return g.omega, g.count, g.cliques.tolist(), g.truncated


def _gather_trunc_body(rank, world):
    # rank 1 is truncated but below the global omega: its list is dropped, so
    # the result is not truncated; max_cliques caps the merged list
    if rank == 0:
        r = Result(3, 3, np.array([[0, 1, 2], [1, 2, 3], [4, 5, 6]], np.int32), False, [], {})
    else:
        r = Result(2, 9, np.array([[7, 8]], np.int32), True, [], {})
    a = mdist.gather_result(r)
    b = mdist.gather_result(r, max_cliques=2)
    return (a.omega, a.count, a.truncated, len(a.cliques)), (b.omega, b.count, b.truncated, b.cliques.tolist())


def _find_one_body(rank, world):
    r = Result(3, 1, np.array([[9, 10, 11]], np.int32), False, [], {}) if rank == 1 else \
        Result(2, 1, np.array([[0, 1]], np.int32), False, [], {})
    g = mdist.gather_result(r, find_one=True)
    return g.omega, g.count, g.cliques.tolist()


def test_bound_sync_is_a_max_allreduce():
    out = spawn(_bound_sync_body)
    for b1, b2 in out:
        assert b1 == (7, 1)  # global best, someone still active
        assert b2 == (6, 0)


def test_gather_adds_multiplicities_and_sorts():
    out = spawn(_gather_body)
    for omega, count, cliques, trunc in out:
        assert omega == 3 and count == 3 and not trunc
        assert cliques == [[0, 1, 2], [1, 2, 3], [4, 5, 6]]


def test_gather_drops_smaller_local_results():
    out = spawn(_gather_mixed_omega_body)
    for omega, count, cliques, trunc in out:
        assert omega == 4 and count == 1 and cliques == [[5, 6, 7, 8]] and trunc


def test_gather_truncation_only_from_omega_holders():
    out = spawn(_gather_trunc_body)
    for a, b in out:
        assert a == (3, 3, False, 3)
        assert b == (3, 3, True, [[0, 1, 2], [1, 2, 3]])


def _sync_raises_body(rank, world):
    """A failing exchange must surface as a Python exception through the
    ctypes callback wrapper (make_options), not a hang or a silent 0."""
    from paper_conf_ipps_geilpo23_b200 import api

    calls = []

    def bad(best, active):
        calls.append(best)
        raise ConnectionError("peer gone")

    o, keep = api.make_options(bound_sync=bad)
    ga = (api.ctypes.c_int32 * 1)(1)
    ret = o.bound_sync(5, 1, ga, None)
    try:
        keep.reraise()
    except ConnectionError as e:
        return ret, ga[0], str(e), len(calls)
    return ret, ga[0], None, len(calls)


def test_bound_sync_exception_is_reported():
    for ret, ga, err, n in spawn(_sync_raises_body):
        assert ret == -1 and ga == 0 and err == "peer gone" and n == 1


def test_find_one_gather_takes_a_holder_of_omega():
    out = spawn(_find_one_body)
    for omega, count, cliques in out:
        assert omega == 3 and count == 1 and cliques == [[9, 10, 11]]


class _FakeGraph:
    """Stands in for a graph handle in agree_core's host logic (CPU, gloo):
    rank 0 "peels" (fills known cores and a peel order), the others record
    what they are given."""

    def __init__(self, n, rank):
        self.n, self.rank, self.device = n, rank, 0
        self.calls = []

    def core_into(self, core, peel):
        self.calls.append("core_into")
        core.copy_(torch.arange(self.n, dtype=torch.int32) % 5)
        peel.copy_(torch.arange(self.n - 1, -1, -1, dtype=torch.int32))

    def set_core(self, core, peel):
        self.calls.append(("set_core", core.tolist(), peel.tolist()))


def _agree_core_body(rank, world):
    g = _FakeGraph(7, rank)
    mdist.agree_core(g)
    opts = {}
    mdist._agree(g, None, world, opts)  # default orientation: agree again
    det = {"orientation": "degeneracy_det"}
    mdist._agree(g, None, world, det)   # the deterministic order: no broadcast
    deg = {"orientation": "degree"}
    mdist._agree(g, None, world, deg)   # the degree order: no broadcast
    return g.calls, opts


def test_agree_core_broadcasts_rank0_cores_and_order():
    """Multi-GPU orientation (distributed.agree_core): rank 0 peels once; every
    other rank receives exactly its core numbers and peel order through one
    broadcast and installs them (mce_set_core), for the degeneracy orientation
    only."""
    out = spawn(_agree_core_body)
    want = ("set_core", [i % 5 for i in range(7)], list(range(6, -1, -1)))
    calls0, opts0 = out[0]
    calls1, opts1 = out[1]
    assert calls0 == ["core_into", "core_into"]
    assert calls1 == [want, want]
    assert opts0 == opts1 == {"orientation": "degeneracy"}


def test_cyclic_deal_partitions_every_root():
    for world in (1, 2, 3, 8):
        for count in (0, 1, 7, 100):
            seen = sorted(i for r in range(world) for i in mdist.owned(count, r, world))
            assert seen == list(range(count))
            assert all(mdist.shard_of(i, world) == r for r in range(world) for i in mdist.owned(count, r, world))


# --- the library's sharding, on one GPU ------------------------------------

@pytest.mark.gpu
@pytest.mark.parametrize("depth", [0, 2, 3, 5])
@pytest.mark.parametrize("shards", [2, 3])
@pytest.mark.parametrize("key", ["planted", "RMAT11", "T(30,6)", "ER400d", "er2000", "BA5k", "BA3k_m2"])
def test_shards_union_is_the_full_answer(key, shards, depth):
    """Each shard enumerates its cyclic share of the roots (depth 0) or, with
    shard_depth d >= 2, every root down to level d - 1 and its hash share of
    the level-d candidates (heuristic seeds dealt either way); merged like
    gather_result, the shards give the oracle's answer."""
    # (BA5k, 3 shards, depth 3) was the round-1 double report: completions above
    # the split fired on one shard's bound and not another's (fixed: none above it)
    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m

    g = GRAPHS[key]()
    om, cl = oracle.max_cliques(*g.numpy())
    gg = m.Graph(g.rowptr, g.col)
    parts = [gg.enumerate(shard_rank=r, shard_count=shards, shard_depth=depth) for r in range(shards)]
    gg.close()
    omega = max(p.omega for p in parts)
    count = sum(p.count for p in parts if p.omega == omega)
    rows = np.concatenate([p.cliques for p in parts if p.omega == omega], 0)
    rows = rows[np.lexsort(rows.T[::-1])]
    assert omega == om and count == len(cl) and np.array_equal(rows, cl)


@pytest.mark.gpu
def test_bound_sync_callback_is_called_every_step():
    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m

    g = GRAPHS["planted"]()
    om, cl = oracle.max_cliques(*g.numpy())
    calls = []

    def sync(best, active):
        calls.append((best, active))
        return best, 0  # a single rank: the global state is the local one

    gg = m.Graph(g.rowptr, g.col)
    r = gg.enumerate(shard_rank=0, shard_count=1, bound_sync=sync)
    gg.close()
    assert r.omega == om and r.count == len(cl) and np.array_equal(r.cliques, cl)
    assert len(calls) >= 2 and calls[-1][1] == 0


@pytest.mark.gpu
@pytest.mark.parametrize("depth", [0, 3])
@pytest.mark.parametrize("key", ["RMAT13", "planted", "ER400d", "T(30,6)"])
def test_shards_on_separate_handles_agree_after_set_order(key, depth):
    """Each "rank" has its own graph handle (its own, possibly different, k-core
    peel order); after mce_set_order with handle 0's order the shards still
    partition the maximum cliques exactly (agree_orientation)."""
    import torch

    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m

    g = GRAPHS[key]()
    om, cl = oracle.max_cliques(*g.numpy())
    shards = 2
    hs = [m.Graph(g.rowptr, g.col) for _ in range(shards)]
    order = hs[0].order_into(torch.empty(g.n, dtype=torch.int32, device="cuda"))
    for h in hs[1:]:
        h.set_order(order)
    o2 = hs[1].order_into(torch.empty(g.n, dtype=torch.int32, device="cuda"))
    assert torch.equal(order, o2)
    parts = [h.enumerate(shard_rank=r, shard_count=shards, shard_depth=depth) for r, h in enumerate(hs)]
    for h in hs:
        h.close()
    omega = max(p.omega for p in parts)
    count = sum(p.count for p in parts if p.omega == omega)
    rows = np.concatenate([p.cliques for p in parts if p.omega == omega], 0)
    rows = rows[np.lexsort(rows.T[::-1])]
    assert omega == om and count == len(cl) and np.array_equal(rows, cl)


@pytest.mark.gpu
@pytest.mark.parametrize("where", ["device", "host"])
@pytest.mark.parametrize("depth", [0, 3])
@pytest.mark.parametrize("key", ["RMAT13", "planted", "BA5k", "T(30,6)"])
def test_shards_on_separate_handles_agree_after_set_core(key, depth, where):
    """Handle 0 peels; the others take its core numbers and peel order with
    mce_set_core (no peel of their own, distributed.agree_core): they orient
    identically, report the same cores and degeneracy, and their shards
    partition the maximum cliques exactly."""
    import torch

    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m
    from paper_conf_ipps_geilpo23_b200 import _lib

    g = GRAPHS[key]()
    om, cl = oracle.max_cliques(*g.numpy())
    shards = 3
    hs = [m.Graph(g.rowptr, g.col) for _ in range(shards)]
    dev = "cuda" if where == "device" else "cpu"
    core = torch.empty(g.n, dtype=torch.int32, device=dev)
    peel = torch.empty(g.n, dtype=torch.int32, device=dev)
    hs[0].core_into(core, peel)
    for h in hs[1:]:
        h.set_core(core, peel)
    c0, o0, d0 = hs[0].preprocess()
    for h in hs[1:]:
        c1, o1, d1 = h.preprocess()
        assert np.array_equal(c0, c1) and np.array_equal(o0, o1) and d0 == d1
    assert d0 == int(c0.max())
    assert _lib.lib().mce_set_core(hs[1]._h, None, None, _lib.WHERE_HOST) == 1  # MCE_ERR_INVALID
    parts = [h.enumerate(shard_rank=r, shard_count=shards, shard_depth=depth) for r, h in enumerate(hs)]
    for h in hs:
        h.close()
    omega = max(p.omega for p in parts)
    count = sum(p.count for p in parts if p.omega == omega)
    rows = np.concatenate([p.cliques for p in parts if p.omega == omega], 0)
    rows = rows[np.lexsort(rows.T[::-1])]
    assert omega == om and count == len(cl) and np.array_equal(rows, cl)


@pytest.mark.gpu
@pytest.mark.parametrize("depth", [0, 2, 3])
@pytest.mark.parametrize("key", ["planted", "RMAT13", "BA5k", "T(30,6)", "ER400d", "RMAT11"])
def test_shards_with_different_bounds(key, depth, monkeypatch):
    """Shards whose lower bounds differ (one with no heuristic and no bound,
    one told omega, one told omega - 1) still partition the maximum cliques
    exactly: nothing reported twice, nothing lost (pre-split
    reporting must not depend on the shard's bound)."""
    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m

    g = GRAPHS[key]()
    om, cl = oracle.max_cliques(*g.numpy(), bound="plain")
    settings = [dict(heuristic="none"), dict(lower_bound=om), dict(lower_bound=max(om - 1, 0), heuristic="single_degree")]
    if depth == 3:  # re-rooted spaces above the split on every level (hash on vertex ids, not local indices)
        monkeypatch.setenv("MCE_REROOT_MIN_W", "1")
    gg = m.Graph(g.rowptr, g.col)
    for shards in (2, 3):
        parts = [gg.enumerate(shard_rank=r, shard_count=shards, shard_depth=depth, **settings[r % 3])
                 for r in range(shards)]
        omega = max(p.omega for p in parts)
        count = sum(p.count for p in parts if p.omega == omega)
        rows = np.concatenate([p.cliques for p in parts if p.omega == omega], 0)
        rows = rows[np.lexsort(rows.T[::-1])]
        assert omega == om and count == len(cl) and np.array_equal(rows, cl), (shards, omega, count)
    gg.close()


@pytest.mark.gpu
@pytest.mark.parametrize("key", ["RMAT13", "BA5k", "planted", "ER400d", "RMAT15"])
def test_deterministic_orientation(key):
    """MCE_ORIENT_DEGENERACY_DET: two handles (two processes' worth of state)
    compute the same order, bit for bit, and it is a degeneracy order
    (out-degree <= core number, checked against the oracle's cores)."""
    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m

    g = GRAPHS[key]()
    rp, col = g.numpy()
    core_o, _, d_o = oracle.core_numbers(rp, col)
    orders = []
    for _ in range(2):
        h = m.Graph(g.rowptr, g.col)
        core, order, d = h.preprocess("degeneracy_det")
        h.close()
        assert np.array_equal(core, core_o) and d == d_o
        orders.append(order)
    assert np.array_equal(orders[0], orders[1])
    order = orders[0]
    assert sorted(order.tolist()) == list(range(g.n))
    rank = np.empty(g.n, np.int64)
    rank[order] = np.arange(g.n)
    src = np.repeat(np.arange(g.n), np.diff(rp))
    up = rank[col] > rank[src]
    assert np.all(np.bincount(src[up], minlength=g.n) <= core_o)
    # cores never decrease along the order
    assert np.all(np.diff(core_o[order]) >= 0)


def _enumerate_mp_body(rank, world):
    import oracle
    from tests.test_gpu_parity import GRAPHS

    import paper_conf_ipps_geilpo23_b200 as m

    out = []
    for key in ("planted", "RMAT13", "BA5k", "ER400d"):
        g = GRAPHS[key]()
        om, cl = oracle.max_cliques(*g.numpy(), bound="plain")
        gg = m.Graph(g.rowptr.cuda(), g.col.cuda())
        for depth in (0, 3):
            gg.clear_cache()
            r = mdist.enumerate_distributed(gg, shard_depth=depth)
            ok = r.omega == om and r.count == len(cl) and np.array_equal(r.cliques, cl)
            f = mdist.find_one_distributed(gg, window=8, shard_depth=depth)
            okf = f.omega == om and oracle.is_clique(*g.numpy(), f.cliques[0])
            out.append((key, depth, bool(ok), bool(okf), r.omega, r.count))
        gg.clear_cache()
        r = mdist.enumerate_distributed(gg, orientation="degeneracy_det")
        ok = r.omega == om and r.count == len(cl) and np.array_equal(r.cliques, cl)
        out.append((key, "det", bool(ok), True, r.omega, r.count))
        gg.close()
    return out


@pytest.mark.gpu
def test_enumerate_distributed_end_to_end():
    """Two processes (gloo process group, both on cuda:0) run the whole
    sharded path -- rank 0's cores and peel order broadcast and set on the
    other rank (agree_core; and the deterministic orientation computed by
    each rank, orientation="degeneracy_det"), cyclic
    root deal or level-3 hash deal, per-step bound all-reduce, final gather --
    and get the oracle's answer (PAPER.md IV-E line 146: root subsets are
    independent)."""
    for rank_out in spawn(_enumerate_mp_body, timeout=900):
        for key, depth, ok, okf, om, cnt in rank_out:
            assert ok and okf, (key, depth, om, cnt)


@pytest.mark.gpu
@pytest.mark.parametrize("config", ["er2000", "ba1m"])
def test_bench_two_ranks(config):
    """bench.py's N > 1 path (torchrun, two ranks; on this one-GPU box both on
    cuda:0 with gloo, the test hooks MCE_BENCH_SAME_DEVICE / MCE_BENCH_BACKEND):
    rank 0 prints one JSON line whose omega and multiplicity equal a one-GPU
    run of the library on the same seeded graph."""
    import json
    import subprocess
    import sys

    import paper_conf_ipps_geilpo23_b200 as m
    from synth import graphs as G

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MCE_BENCH_SAME_DEVICE="1", MCE_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2",
           "--steps", "3", "--warmup", "3", "--config", config, "--no-cpu-baseline"]
    out = subprocess.run(cmd, cwd=root, env=env, capture_output=True, text=True, timeout=900)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    rec = json.loads(lines[0])
    assert rec["n_gpus"] == 2 and rec["value"] > 0
    g = G.make_config(config)
    gg = m.Graph(g.rowptr.cuda(), g.col.cuda())
    r = gg.enumerate()
    gg.close()
    assert rec["details"]["omega"] == r.omega and rec["details"]["multiplicity"] == r.count
