"""The shared seeded generators: counter RNG pinned to pure-Python SplitMix64,
CSR well-formedness, and the shapes of the BASELINE.json workloads."""

import numpy as np
import pytest
import torch

from synth import graphs as G


def test_splitmix_matches_python():
    xs = [0, 1, 2**63 - 1, 2**63, 2**64 - 1, 12345678901234567, 0xDEADBEEF]
    t = torch.tensor([G._s64(x) for x in xs], dtype=torch.int64)
    got = [v & G._M64 for v in G.splitmix64(t).tolist()]
    assert got == [G.splitmix64_py(x) for x in xs]


def _check_csr(g):
    rp, col = g.numpy()
    assert rp[0] == 0 and rp[-1] == col.size and np.all(np.diff(rp) >= 0)
    src = np.repeat(np.arange(g.n), np.diff(rp))
    assert np.all(src != col)  # no loops
    for v in range(min(g.n, 200)):
        nb = col[rp[v]:rp[v + 1]]
        assert np.all(np.diff(nb) > 0)  # sorted, no duplicates
    e = set(zip(src.tolist(), col.tolist()))
    assert all((b, a) in e for a, b in list(e)[:5000])  # symmetric


@pytest.mark.parametrize("maker", [
    lambda: G.erdos_renyi(300, 0.05, seed=3),
    lambda: G.rmat(10, 8, 0.57, 0.19, 0.19, seed=2),
    lambda: G.barabasi_albert(500, 4, seed=1),
    lambda: G.turan_graph(11, 3),
    lambda: G.paley_graph(13),
])
def test_csr_wellformed(maker):
    _check_csr(maker())


def test_deterministic():
    a = G.rmat(9, 8, 0.57, 0.19, 0.19, seed=5)
    b = G.rmat(9, 8, 0.57, 0.19, 0.19, seed=5, chunk=1000)
    assert torch.equal(a.rowptr, b.rowptr) and torch.equal(a.col, b.col)
    c = G.rmat(9, 8, 0.57, 0.19, 0.19, seed=6)
    assert not torch.equal(a.col, c.col) or not torch.equal(a.rowptr, c.rowptr)


def test_ba_shape():
    g = G.barabasi_albert(2000, 4, seed=1)
    assert g.num_edges == 4 * (2000 - 4)  # m distinct targets per new vertex
    deg = np.diff(g.numpy()[0])
    assert deg[4:].min() >= 4


def test_planted():
    g = G.plant_cliques(G.erdos_renyi(400, 0.01, seed=1), 3, 7, seed=9)
    rp, col = g.numpy()
    assert len(g.planted) == 3
    seen = set()
    for c in g.planted:
        assert len(c) == 7 and not (seen & set(c))
        seen |= set(c)
        for i in c:
            nb = set(col[rp[i]:rp[i + 1]].tolist())
            assert set(c) - {i} <= nb
