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
BOUNDS = ["size", "color", "plain", "plain_id"]  # oracle_mce (two bounds), oracle_mce_plain (two orders)


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


@pytest.mark.parametrize("bound", BOUNDS)
def test_lower_bound_does_not_change_answer(bound):
    edges = random_small_graph(16, 0.6, 7)
    rp, col = csr_from_edges(16, edges)
    om, cl = oracle.max_cliques(rp, col)
    for lb in range(0, om + 1):
        om2, cl2 = oracle.max_cliques(rp, col, lb=lb, bound=bound)
        assert om2 == om and cl2.tolist() == cl.tolist()
    # a lower bound above omega: nothing of that size exists
    om3, cl3 = oracle.max_cliques(rp, col, lb=om + 1, bound=bound)
    assert om3 == 0 and cl3.shape[0] == 0


# ---------------------------------------------------------------------------
# closed forms
# ---------------------------------------------------------------------------


@pytest.mark.parametrize("bound", BOUNDS)
@pytest.mark.parametrize("n", [1, 2, 3, 5, 9, 16])
def test_complete_graph(n, bound):
    g = G.complete_graph(n)
    om, cl = oracle.max_cliques(*g.numpy(), bound=bound)
    assert om == n and cl.tolist() == [list(range(n))]
    assert oracle.count_max_cliques(*g.numpy(), bound=bound) == (n, 1)
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


# ---------------------------------------------------------------------------
# the two oracles against each other, and the multi-word (out-degree > 64)
# bitset path of oracle_mce against closed forms
# ---------------------------------------------------------------------------

# graphs of the GPU parity set the list-based oracle finishes in < 1 s
CROSS = {
    "ER60": lambda: G.erdos_renyi(60, 0.3, seed=4),
    "ER300": lambda: G.erdos_renyi(300, 0.1, seed=5),
    "ER150d": lambda: G.erdos_renyi(150, 0.5, seed=6),
    "ER400d": lambda: G.erdos_renyi(400, 0.35, seed=7),
    "RMAT11": lambda: G.rmat(11, 8, 0.57, 0.19, 0.19, seed=3),
    "RMAT13": lambda: G.rmat(13, 8, 0.45, 0.2, 0.2, seed=2),
    "BA5k": lambda: G.barabasi_albert(5000, 4, seed=2),
    "BA3k_m1": lambda: G.barabasi_albert(3000, 1, seed=11),
    "planted": lambda: G.plant_cliques(G.erdos_renyi(3000, 0.004, seed=9), 3, 9, seed=9),
    "T(36,12)": lambda: G.turan_graph(36, 12),
    # out-degree > 64 after orientation: oracle_mce's multi-word bitsets
    "ER200x": lambda: G.erdos_renyi(200, 0.5, seed=3),  # degeneracy 84, W = 2
    "ER150x": lambda: G.erdos_renyi(150, 0.6, seed=3),  # degeneracy 77, 96 maximum cliques
    "ER300x": lambda: G.erdos_renyi(300, 0.4, seed=3),  # degeneracy 101
}


@pytest.mark.parametrize("key", list(CROSS))
def test_colour_oracle_vs_plain_oracle(key):
    """oracle_mce (degeneracy order, root-local bitsets, colouring bound) and
    oracle_mce_plain (degree order, sorted lists, |C|+|P| bound) share no
    search code: they must agree clique for clique."""
    rp, col = CROSS[key]().numpy()
    om, cl = oracle.max_cliques(rp, col, bound="color")
    om_p, cl_p = oracle.max_cliques(rp, col, bound="plain")
    assert om == om_p and np.array_equal(cl, cl_p)
    om_t, cl_t = oracle.max_cliques(rp, col, bound="color", tight=True)
    assert om_t == om and np.array_equal(cl_t, cl)
    assert oracle.count_max_cliques(rp, col, bound="color", tight=True) == (om, len(cl))
    assert oracle.count_max_cliques(rp, col, bound="plain") == (om, len(cl))
    # invariants: cliques of size omega, none bigger
    for c in cl[:50]:
        assert oracle.is_clique(rp, col, c)
    kc = oracle.kclique_counts(rp, col, om + 1) if key not in ("T(36,12)",) else None
    if kc is not None:
        assert kc[om - 1] == len(cl) and kc[om] == 0


@pytest.mark.parametrize("bound", ["size", "color", "plain"])
@pytest.mark.parametrize("n", [65, 130, 300])
def test_complete_graph_multiword(n, bound):
    """K_n with n - 1 > 64 later neighbours at the root: W = 2, 3, 5 words."""
    om, cl = oracle.max_cliques(*G.complete_graph(n).numpy(), bound=bound)
    assert om == n and cl.tolist() == [list(range(n))]


@pytest.mark.parametrize("tight", [False, True])
@pytest.mark.parametrize("j,t", [(3, 1), (13, 5), (6, 60), (12, 300), (16, 50), (8, 600)])
def test_cocktail_party_join_closed_form(j, t, tight):
    """CP(j) + K_t: omega = j + t, exactly 2^j maximum cliques, each taking
    one vertex of every non-adjacent pair.  (8, 600): root out-degree 615,
    the (512, 1024] width class of R-MAT scale 22/26 roots."""
    g = G.cocktail_party_join(j, t, seed=j * 1000 + t)
    rp, col = g.numpy()
    om, cl = oracle.max_cliques(rp, col, tight=tight)
    assert om == j + t and len(cl) == 2 ** j
    assert len({tuple(c) for c in cl}) == len(cl)
    deg = np.diff(rp)
    # the non-adjacent pairs are the only vertices of degree n - 2
    paired = set(np.nonzero(deg == g.n - 2)[0].tolist())
    assert len(paired) == 2 * j
    for c in cl[:64]:
        assert len(set(c.tolist()) & paired) == j  # one of each pair
        assert oracle.is_clique(rp, col, c)
    assert oracle.count_max_cliques(rp, col, tight=tight) == (j + t, 2 ** j)


def test_turan_multiword():
    """T(150, 3): parts of 50, out-degree up to 100 (W = 2), 50^3 maximum cliques."""
    rp, col = G.turan_graph(150, 3).numpy()
    for bound in ("color", "plain"):
        assert oracle.count_max_cliques(rp, col, bound=bound) == (3, 125000)


def test_is_clique_negative():
    """oracle_is_clique must reject non-cliques (every find-one check relies on it)."""
    g = G.cocktail_party_join(4, 6, seed=1)
    rp, col = g.numpy()
    deg = np.diff(rp)
    paired = np.nonzero(deg == g.n - 2)[0]
    a = int(paired[0])
    row = set(col[rp[a]:rp[a + 1]].tolist())
    b = next(int(v) for v in paired if int(v) != a and int(v) not in row)  # a's non-neighbour
    others = [v for v in range(g.n) if v not in set(paired.tolist())]  # the K_t part: adjacent to all
    assert not oracle.is_clique(rp, col, [a, b])
    assert not oracle.is_clique(rp, col, others[:5] + [a, b])
    assert not oracle.is_clique(rp, col, [b] + others[:3] + [a])
    assert oracle.is_clique(rp, col, [a] + others[:5])
    assert oracle.is_clique(rp, col, [a])
    assert oracle.is_clique(rp, col, [])
    # against brute force on every subset of a small random graph
    edges = random_small_graph(9, 0.5, 3)
    rp2, col2 = csr_from_edges(9, edges)
    es = {tuple(e) for e in edges}
    for mask in range(1 << 9):
        vs = [v for v in range(9) if mask >> v & 1]
        truth = all((u, w) in es for u, w in combinations(vs, 2))
        assert oracle.is_clique(rp2, col2, vs) == truth
