"""Pins for the CPU oracle (oracle/) against things other than itself.

Every check here compares the oracle with brute force, a closed form, a
hand-traced fixture, or an invariant that follows from the definition of a
maximum clique (PAPER.md II line 47) -- never with the oracle's own formula.
"""

import json
import math
import os
from itertools import combinations

import numpy as np
import pytest
import torch

import oracle
from synth import graphs as G
from tests import bruteforce as bf

HERE = os.path.dirname(os.path.abspath(__file__))
BOUNDS = ["size", "color"]


def csr_from_edges(n, edges):
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    g = G.from_edges(n, torch.from_numpy(e[:, 0].copy()), torch.from_numpy(e[:, 1].copy()))
    return g.numpy()


def random_small_graph(n, p, seed):
    rng = np.random.default_rng(seed)
    edges = [(u, v) for u in range(n) for v in range(u + 1, n) if rng.random() < p]
    return edges


# ---------------------------------------------------------------------------
# brute force (n <= 18)
# ---------------------------------------------------------------------------


@pytest.mark.parametrize("bound", BOUNDS)
@pytest.mark.parametrize("seed", range(12))
def test_max_cliques_vs_bruteforce(seed, bound):
    n = 6 + seed % 12
    p = [0.2, 0.5, 0.8][seed % 3]
    edges = random_small_graph(n, p, seed)
    rp, col = csr_from_edges(n, edges)
    om, cl = oracle.max_cliques(rp, col, bound=bound)
    bom, bcl = bf.max_cliques(n, edges)
    assert om == bom
    assert cl.tolist() == bcl


@pytest.mark.parametrize("seed", range(6))
def test_kclique_counts_vs_bruteforce(seed):
    n = 8 + seed
    edges = random_small_graph(n, 0.6, 100 + seed)
    rp, col = csr_from_edges(n, edges)
    assert oracle.kclique_counts(rp, col, n).tolist() == bf.kclique_counts(n, edges, n)


@pytest.mark.parametrize("seed", range(6))
def test_core_numbers_vs_definition(seed):
    n = 10 + 3 * seed
    edges = random_small_graph(n, 0.3, 200 + seed)
    rp, col = csr_from_edges(n, edges)
    core, order, d = oracle.core_numbers(rp, col)
    assert core.tolist() == bf.core_numbers_by_definition(n, edges)
    assert d == max(core.tolist() + [0])
    assert sorted(order.tolist()) == list(range(n))


def test_lower_bound_does_not_change_answer():
    edges = random_small_graph(16, 0.6, 7)
    rp, col = csr_from_edges(16, edges)
    om, cl = oracle.max_cliques(rp, col)
    for lb in range(0, om + 1):
        om2, cl2 = oracle.max_cliques(rp, col, lb=lb)
        assert om2 == om and cl2.tolist() == cl.tolist()


# ---------------------------------------------------------------------------
# closed forms
# ---------------------------------------------------------------------------


@pytest.mark.parametrize("bound", BOUNDS)
@pytest.mark.parametrize("n", [1, 2, 3, 5, 9, 16])
def test_complete_graph(n, bound):
    g = G.complete_graph(n)
    om, cl = oracle.max_cliques(*g.numpy(), bound=bound)
    assert om == n and cl.tolist() == [list(range(n))]
    counts = oracle.kclique_counts(*g.numpy(), n + 1)
    assert counts.tolist() == [math.comb(n, k) for k in range(1, n + 2)]


@pytest.mark.parametrize("bound", BOUNDS)
@pytest.mark.parametrize("n", [4, 5, 6, 11])
def test_cycle(n, bound):
    g = G.cycle_graph(n)
    om, cl = oracle.max_cliques(*g.numpy(), bound=bound)
    assert om == 2 and len(cl) == n  # C_5: omega 2, multiplicity 5


@pytest.mark.parametrize("bound", BOUNDS)
@pytest.mark.parametrize("n,k", [(6, 3), (9, 3), (10, 4), (12, 4), (13, 5), (15, 5)])
def test_turan(n, k, bound):
    g = G.turan_graph(n, k)
    parts = [len(range(r, n, k)) for r in range(k)]
    om, cl = oracle.max_cliques(*g.numpy(), bound=bound)
    assert om == k
    assert len(cl) == math.prod(parts)
    # k-cliques of T(n,k): elementary symmetric polynomials of the part sizes
    counts = oracle.kclique_counts(*g.numpy(), k + 1)
    for j in range(1, k + 2):
        e_j = sum(math.prod(c) for c in combinations(parts, j))
        assert counts[j - 1] == e_j


@pytest.mark.parametrize("bound", BOUNDS)
@pytest.mark.parametrize("q", [5, 13, 17])
def test_paley(q, bound):
    """Paley(q) is srg(q, (q-1)/2, (q-5)/4, (q-1)/4): q(q-1)(q-5)/48 triangles.
    P(5) = C_5; P(13) and P(17) have no K4 (P(17) is the R(4,4) > 17 witness)."""
    g = G.paley_graph(q)
    om, cl = oracle.max_cliques(*g.numpy(), bound=bound)
    if q == 5:
        assert om == 2 and len(cl) == 5
    else:
        assert om == 3 and len(cl) == q * (q - 1) * (q - 5) // 48


def test_null_and_edgeless():
    om, cl = oracle.max_cliques(np.zeros(1, np.int64), np.zeros(0, np.int32))
    assert om == 0 and cl.shape == (1, 0)
    om, cl = oracle.max_cliques(np.zeros(6, np.int64), np.zeros(0, np.int32))
    assert om == 1 and cl.tolist() == [[v] for v in range(5)]


def test_planted_clique_sparse():
    g = G.make_config("er2000")  # G(2000, 0.005) + planted 12-clique (configs[0])
    om, cl = oracle.max_cliques(*g.numpy())
    assert om == 12 and cl.tolist() == g.planted
    w, runs, best = oracle.greedy(*g.numpy(), threshold=np.diff(g.numpy()[0]), h=g.n)
    assert w <= om


def test_disjoint_union_multiplicity():
    """omega of a disjoint union is the max; multiplicity adds (closed form)."""
    parts = [G.complete_graph(5), G.turan_graph(9, 5), G.complete_graph(4)]
    edges, off = [], 0
    for p in parts:
        edges += [(u + off, v + off) for u, v in p.edges()]
        off += p.n
    rp, col = csr_from_edges(off, edges)
    om, cl = oracle.max_cliques(rp, col)
    # K5 -> 1 clique of size 5; T(9,5) parts 2,2,2,2,1 -> 16 cliques of size 5
    assert om == 5 and len(cl) == 1 + 16


# ---------------------------------------------------------------------------
# invariants on random graphs (multiplicity == number of omega-cliques)
# ---------------------------------------------------------------------------


@pytest.mark.parametrize("seed", range(4))
def test_invariants_random(seed):
    g = G.erdos_renyi(120, 0.25, seed=seed)
    rp, col = g.numpy()
    om, cl = oracle.max_cliques(rp, col)
    assert len({tuple(c) for c in cl}) == len(cl)  # no duplicates
    for c in cl:
        assert oracle.is_clique(rp, col, c)
    counts = oracle.kclique_counts(rp, col, om + 1)
    assert counts[om - 1] == len(cl)  # every omega-clique listed
    assert counts[om] == 0  # no (omega+1)-clique exists
    om_s, cl_s = oracle.max_cliques(rp, col, bound="size")
    assert om_s == om and cl_s.tolist() == cl.tolist()


# ---------------------------------------------------------------------------
# greedy heuristic: hand-traced fixture
# ---------------------------------------------------------------------------


def _trace():
    with open(os.path.join(HERE, "golden", "greedy_trace.json")) as f:
        return json.load(f)


def test_greedy_trace_degree():
    t = _trace()
    rp, col = csr_from_edges(t["n"], t["edges"])
    deg = np.diff(rp)
    w, runs, best = oracle.greedy(rp, col, deg, t["n"])
    assert runs.tolist() == t["degree"]["run_sizes"]
    assert best.tolist() == t["degree"]["best_clique"]
    for h, expect in t["degree"]["omega_bar_by_h"].items():
        assert oracle.greedy(rp, col, deg, int(h))[0] == expect


def test_greedy_trace_core():
    t = _trace()
    rp, col = csr_from_edges(t["n"], t["edges"])
    core, _, _ = oracle.core_numbers(rp, col)
    assert core.tolist() == t["core"]["core_numbers"]
    w, runs, best = oracle.greedy(rp, col, core, t["n"])
    assert runs.tolist() == t["core"]["run_sizes"]
    assert best.tolist() == t["core"]["best_clique"]
    for h, expect in t["core"]["omega_bar_by_h"].items():
        assert oracle.greedy(rp, col, core, int(h))[0] == expect


def test_trace_graph_cliques():
    t = _trace()
    rp, col = csr_from_edges(t["n"], t["edges"])
    assert oracle.kclique_counts(rp, col, 5).tolist() == t["kclique_counts"]
    om, cl = oracle.max_cliques(rp, col)
    assert om == t["omega"] and cl.tolist() == t["max_cliques"]


@pytest.mark.parametrize("seed", range(4))
def test_greedy_properties(seed):
    g = G.erdos_renyi(200, 0.1, seed=50 + seed)
    rp, col = g.numpy()
    om, _ = oracle.max_cliques(rp, col)
    for thr in (np.diff(rp), oracle.core_numbers(rp, col)[0]):
        w, runs, best = oracle.greedy(rp, col, thr, g.n)
        assert 1 <= w <= om
        assert len(best) == w and oracle.is_clique(rp, col, best)
        assert runs.max() == w
        # the multi-run bound is at least the single-run bound (max over more runs)
        assert w >= oracle.greedy(rp, col, thr, 1)[0]


def test_greedy_closed_forms():
    for n in (1, 4, 9):
        g = G.complete_graph(n)
        rp, col = g.numpy()
        assert oracle.greedy(rp, col, np.diff(rp), 1)[0] == n
    g = G.turan_graph(12, 4)  # every maximal clique of T(n,k) has k vertices
    rp, col = g.numpy()
    w, runs, _ = oracle.greedy(rp, col, np.diff(rp), g.n)
    assert w == 4 and set(runs.tolist()) == {4}
