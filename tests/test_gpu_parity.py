"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bit-exact for everything (omega, multiplicity, the sorted list of sorted
cliques, core numbers, greedy run sizes); find_one returns a clique whose
size equals the oracle's omega (several answers are correct there, so the
rest is checked for validity).
"""

import functools
import json
import os

import numpy as np
import pytest
import torch

import oracle
from synth import graphs as G
from tests import bruteforce as bf

pytestmark = pytest.mark.gpu


def mce():
    import paper_conf_ipps_geilpo23_b200 as m

    return m


# The parity reference is the list-based oracle (oracle_mce_plain: PAPER.md
# II-A with the |C|+|P| bound, no bitsets, no colouring -- nothing shared with
# the kernels' layout) wherever it finishes in seconds; the colouring oracle
# (pinned against it and against closed forms in tests/test_oracle.py) only
# where the |C|+|P| bound alone is exponential (R-MAT hub cores, CP(j)+K_t).
COLOUR_ONLY = {"RMAT15", "CP8+K600", "CP12+K300", "ER700w8", "ER1000w8"}


@functools.lru_cache(maxsize=None)
def oracle_answer(key):
    g = GRAPHS[key]()
    om, cl = oracle.max_cliques(*g.numpy(), bound="color" if key in COLOUR_ONLY else "plain")
    return om, cl


GRAPHS = {
    "K1": lambda: G.complete_graph(1),
    "K2": lambda: G.complete_graph(2),
    "K7": lambda: G.complete_graph(7),
    "K64": lambda: G.complete_graph(64),
    "K65": lambda: G.complete_graph(65),
    "K130": lambda: G.complete_graph(130),
    "K257": lambda: G.complete_graph(257),  # a full 4-word candidate set: 256 colours
    "C5": lambda: G.cycle_graph(5),
    "C9": lambda: G.cycle_graph(9),
    "T(12,4)": lambda: G.turan_graph(12, 4),
    "T(30,6)": lambda: G.turan_graph(30, 6),
    "T(36,12)": lambda: G.turan_graph(36, 12),
    "Paley13": lambda: G.paley_graph(13),
    "Paley17": lambda: G.paley_graph(17),
    "ER60": lambda: G.erdos_renyi(60, 0.3, seed=4),
    "ER300": lambda: G.erdos_renyi(300, 0.1, seed=5),
    "ER150d": lambda: G.erdos_renyi(150, 0.5, seed=6),
    "ER400d": lambda: G.erdos_renyi(400, 0.35, seed=7),
    "RMAT11": lambda: G.rmat(11, 8, 0.57, 0.19, 0.19, seed=3),
    "RMAT13": lambda: G.rmat(13, 8, 0.45, 0.2, 0.2, seed=2),
    "RMAT15": lambda: G.rmat(15, 16, 0.57, 0.19, 0.19, seed=5),  # 121 hubs of degree > 1024
    "BA5k": lambda: G.barabasi_albert(5000, 4, seed=2),
    # degeneracy <= 3: every root has |N+(r)| <= 4, the sparse root kernel (root_expand_l4)
    "BA3k_m1": lambda: G.barabasi_albert(3000, 1, seed=11),  # a tree: omega 2, every edge maximum
    "BA3k_m2": lambda: G.barabasi_albert(3000, 2, seed=11),
    "BA3k_m3": lambda: G.barabasi_albert(3000, 3, seed=11),
    "planted": lambda: G.plant_cliques(G.erdos_renyi(3000, 0.004, seed=9), 3, 9, seed=9),
    "er2000": lambda: G.make_config("er2000"),
    # root out-degree 615: the (512, 1024] width class (W = 16) of the R-MAT scale 22 / 26 roots
    "CP8+K600": lambda: G.cocktail_party_join(8, 600, seed=8600),
    "CP12+K300": lambda: G.cocktail_party_join(12, 300, seed=12300),  # W = 8, 4096 cliques
    # dense, degeneracy 286 / 314: W = 8 roots whose candidates keep many colour
    # classes within the bound (more than the shared-memory kernels' class ring)
    "ER700w8": lambda: G.erdos_renyi(700, 0.45, seed=3),
    "ER1000w8": lambda: G.erdos_renyi(1000, 0.35, seed=2),
}


def run_enum(g, **kw):
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    try:
        return gg.enumerate(**kw)
    finally:
        gg.close()


@pytest.mark.parametrize("legacy_roots", [False, True])
@pytest.mark.parametrize("key", list(GRAPHS))
def test_enumerate_matches_oracle(key, legacy_roots):
    """Fused root-level kernel (default) and the generic per-level path both match the oracle."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    r = run_enum(g, legacy_roots=legacy_roots)
    assert r.omega == om
    assert r.count == len(cl)
    assert np.array_equal(r.cliques, cl)


@pytest.mark.parametrize("key", ["er2000", "planted", "RMAT11", "RMAT13", "K130", "T(30,6)", "ER400d", "Paley17"])
def test_unfused_levels_match(key):
    """Every level through count -> scan -> write launches (no expand_small) gives the same answer."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    r = run_enum(g, fused_levels=False)
    assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)


@pytest.mark.parametrize("key", ["er2000", "planted", "RMAT11", "BA5k", "BA3k_m1", "BA3k_m2", "C9", "T(36,12)"])
def test_no_heuristic_size2_leaves(key):
    """Heuristic 'none' with a lower bound of 2: size-2 leaves come out of the fused root kernel."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    r = run_enum(g, heuristic="none", bound="size" if key == "C9" else "color")
    assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)


def test_triangle_free_many_leaves():
    """omega = 2 with more edges than the initial leaf staging (4096 rows): staging grows, replay is exact."""
    n = 6000
    i = torch.arange(n, dtype=torch.int64)
    g = G.from_edges(n, i, (i + 1) % n)  # C_6000: 6000 maximum cliques of size 2
    r = run_enum(g, heuristic="none")
    assert r.omega == 2 and r.count == n
    rows = np.sort(np.stack([i.numpy(), ((i + 1) % n).numpy()], 1), axis=1)
    rows = rows[np.lexsort(rows.T[::-1])]
    assert np.array_equal(r.cliques, rows.astype(np.int32))


@pytest.mark.parametrize("bound", ["size", "color"])
@pytest.mark.parametrize("orientation", ["degeneracy", "degree"])
@pytest.mark.parametrize("heuristic", ["none", "single_degree", "single_core", "multi_degree", "multi_core"])
@pytest.mark.parametrize("key", ["ER60", "T(12,4)", "Paley17", "RMAT11", "planted"])
def test_option_grid(key, heuristic, orientation, bound):
    if bound == "size" and key in ("RMAT11",):
        pytest.skip("size bound alone is exponential on the R-MAT hub core")
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    r = run_enum(g, heuristic=heuristic, orientation=orientation, bound=bound)
    assert (r.omega, r.count) == (om, len(cl))
    assert np.array_equal(r.cliques, cl)


@pytest.mark.parametrize("seed", range(8))
def test_random_small_vs_bruteforce(seed):
    n = 10 + seed
    rng = np.random.default_rng(seed)
    edges = [(u, v) for u in range(n) for v in range(u + 1, n) if rng.random() < 0.55]
    e = np.asarray(edges, np.int64).reshape(-1, 2)
    g = G.from_edges(n, torch.from_numpy(e[:, 0].copy()), torch.from_numpy(e[:, 1].copy()))
    bom, bcl = bf.max_cliques(n, edges)
    r = run_enum(g)
    assert r.omega == bom and r.cliques.tolist() == bcl


def test_empty_and_edgeless():
    m = mce()
    g = m.Graph(np.zeros(1, np.int64), np.zeros(0, np.int32))
    r = g.enumerate()
    assert r.omega == 0 and r.count == 1
    g = m.Graph(np.zeros(8, np.int64), np.zeros(0, np.int32))
    r = g.enumerate()
    assert r.omega == 1 and r.count == 7 and r.cliques.tolist() == [[v] for v in range(7)]
    r = g.find_one()
    assert r.omega == 1 and r.cliques.shape == (1, 1)


def test_device_input_and_validation():
    m = mce()
    g = GRAPHS["ER300"]()
    gg = m.Graph(g.rowptr.cuda(), g.col.cuda(), validate=True)
    om, cl = oracle_answer("ER300")
    r = gg.enumerate()
    assert r.omega == om and np.array_equal(r.cliques, cl)
    bad_col = g.col.clone()
    bad_col[0], bad_col[1] = bad_col[1].item(), bad_col[0].item()  # unsorted row
    with pytest.raises(m.MCEError):
        m.Graph(g.rowptr, bad_col, validate=True)


@pytest.mark.parametrize("key", ["ER300", "RMAT11", "BA5k", "T(30,6)", "ER400d"])
def test_core_numbers_and_orientation(key):
    g = GRAPHS[key]()
    rp, col = g.numpy()
    core_o, _, d_o = oracle.core_numbers(rp, col)
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    for orientation in ("degeneracy", "degree"):
        gg.clear_cache()
        core, order, d = gg.preprocess(orientation)
        assert np.array_equal(core, core_o) and d == d_o
        assert sorted(order.tolist()) == list(range(g.n))
        rank = np.empty(g.n, np.int64)
        rank[order] = np.arange(g.n)
        src = np.repeat(np.arange(g.n), np.diff(rp))
        up = rank[col] > rank[src]
        outdeg = np.bincount(src[up], minlength=g.n)
        if orientation == "degeneracy":  # a degeneracy order: out-degree <= core number
            assert np.all(outdeg <= core_o)
        else:  # degree order: edges point to vertices of larger or equal degree
            deg = np.diff(rp)
            assert np.all(deg[col[up]] >= deg[src[up]])


@pytest.mark.parametrize("key", ["ER300", "RMAT11", "BA5k", "planted", "ER150d"])
@pytest.mark.parametrize("kind", ["degree", "core"])
def test_heuristic_matches_oracle(key, kind):
    g = GRAPHS[key]()
    rp, col = g.numpy()
    thr = np.diff(rp) if kind == "degree" else oracle.core_numbers(rp, col)[0]
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    order = np.lexsort((np.arange(g.n), -thr.astype(np.int64)))  # seeds: threshold desc, id asc
    for h in (1, 7, g.n):
        w_o, runs_o, best_o = oracle.greedy(rp, col, thr, h)
        w, clique, runs = gg.heuristic(("single_" if h == 1 else "multi_") + kind, h)
        assert w == w_o
        assert clique == best_o.tolist()
        assert np.array_equal(runs[order[:h]], runs_o)
        assert np.count_nonzero(runs) == h


@pytest.mark.parametrize("window", [1, 3, 64, 0])
@pytest.mark.parametrize("key", ["ER300", "planted", "ER400d", "RMAT13", "K130", "T(30,6)"])
def test_find_one(key, window):
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    r = gg.find_one(window=window)
    assert r.omega == om and r.count == 1 and r.cliques.shape == (1, om)
    assert oracle.is_clique(*g.numpy(), r.cliques[0])
    assert len(set(r.cliques[0].tolist())) == om


def test_find_one_turan_closed_form():
    """T(200,20) has 10^20 maximum cliques (omega = 20): only find-one is possible."""
    g = G.turan_graph(200, 20)
    m = mce()
    r = m.Graph(g.rowptr, g.col).find_one(window=16)
    assert r.omega == 20 and sorted(int(v) % 20 for v in r.cliques[0]) == list(range(20))


@pytest.mark.parametrize("key", ["ER400d", "T(30,6)", "RMAT13"])
def test_small_budget_chunking(key):
    """A frontier budget far below the peak level forces chunked (recursive
    windowed) expansion; the answer must not change."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    r = run_enum(g, budget_bytes=4 << 20, heuristic="none")
    assert r.omega == om and np.array_equal(r.cliques, cl)


def test_max_cliques_truncation():
    g = G.turan_graph(24, 6)  # parts of 4: 4^6 = 4096 maximum cliques
    r = run_enum(g, max_cliques=100)
    assert r.omega == 6 and r.count == 4096 and r.truncated and r.cliques.shape == (100, 6)
    for c in r.cliques:
        assert len({int(v) % 6 for v in c}) == 6


@pytest.mark.slow
def test_config_ba1m_full():
    g = G.make_config("ba1m")
    om, cl = oracle.max_cliques(*g.numpy())
    r = run_enum(g)
    assert r.omega == om and np.array_equal(r.cliques, cl)


@pytest.mark.slow
def test_config_dense800_find_one():
    g = G.make_config("dense800")
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    r = gg.find_one(window=32)
    assert r.omega == 15  # tests/golden/dense800.json (oracle, scripts/make_golden.py)
    assert oracle.is_clique(*g.numpy(), r.cliques[0])


@pytest.mark.parametrize("shortcut", [True, False])
@pytest.mark.parametrize("j,t", [(13, 5), (12, 300), (6, 60), (3, 1), (8, 600)])
def test_clique_completions_closed_form(j, t, shortcut):
    """Completions (P a clique, reading 10) on the thread (W <= 4) and
    tile (W >= 8, W = 16 for (8, 600)) kernels: 2^13 > the 4096-row staging
    forces growth + replay."""
    g = G.cocktail_party_join(j, t, seed=j * 1000 + t)
    om, cl = oracle.max_cliques(*g.numpy())
    assert om == j + t and len(cl) == 2 ** j  # closed form pins the oracle here too
    for fused in (True, False):
        r = run_enum(g, clique_shortcut=shortcut, fused_levels=fused)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)
    # a small budget forces chunked levels (the 312-level chain itself needs ~35 MB of parent links)
    r = run_enum(g, clique_shortcut=shortcut, budget_bytes=64 << 20)
    assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)
    m = mce()
    f = m.Graph(g.rowptr, g.col).find_one(window=4)
    assert f.omega == om and oracle.is_clique(*g.numpy(), f.cliques[0])


@pytest.mark.parametrize("key", ["er2000", "planted", "RMAT11", "RMAT13", "K65", "K130", "K257", "T(36,12)", "ER400d",
                                 "Paley17", "BA5k"])
def test_clique_shortcut_off_matches(key):
    """Algorithm 2's level-by-level expansion (no completions) gives the same answer."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    r = run_enum(g, clique_shortcut=False)
    assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)
    r = run_enum(g, clique_shortcut=False, fused_levels=False)
    assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)


@pytest.mark.parametrize("key", ["RMAT15", "RMAT13", "BA5k", "planted"])
def test_heuristic_hub_runs(key):
    """Runs on hub seeds (degree > 1024: block per run) and the exact early abort:
    the bound and the winning clique equal the oracle's; with every run size
    requested nothing is aborted."""
    g = GRAPHS[key]()
    rp, col = g.numpy()
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    w_o, runs_o, best_o = oracle.greedy(rp, col, np.diff(rp), g.n)
    r = gg.enumerate()  # aborting heuristic inside the pipeline
    w, clique, runs = gg.heuristic("multi_degree", g.n)
    assert w == w_o and clique == best_o.tolist()
    order = np.lexsort((np.arange(g.n), -np.diff(rp).astype(np.int64)))
    assert np.array_equal(runs[order], runs_o)
    assert r.omega == oracle_answer(key)[0]


@pytest.mark.parametrize("key", ["er2000", "planted", "RMAT11", "RMAT13", "K130", "K257", "T(30,6)", "ER400d",
                                 "Paley17", "BA5k"])
def test_fused_expand_off_matches(key):
    """The separate count -> scan -> write passes (no fused count + write) give the same answer."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    for fused_levels in (True, False):
        r = run_enum(g, fused_expand=False, fused_levels=fused_levels)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)


@pytest.mark.parametrize("key", ["ER400d", "RMAT13", "T(36,12)"])
def test_fused_expand_overflow(key):
    """A budget too small for a level's children makes the fused pass overflow
    (falls back to scan + chunked writes); find-one under the same budget."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    for budget in (2 << 20, 6 << 20, 32 << 20):
        r = run_enum(g, budget_bytes=budget, heuristic="none", fused_levels=False)
        assert r.omega == om and np.array_equal(r.cliques, cl)


@pytest.mark.parametrize("key", ["er2000", "planted", "RMAT15", "BA5k", "ER400d"])
def test_overlap_off_matches(key):
    """Heuristic after preprocessing (no second stream / thread) gives the same answer."""
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    for heuristic in ("multi_degree", "single_degree"):
        r = run_enum(g, overlap=False, heuristic=heuristic)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)
        m = mce()
        f = m.Graph(g.rowptr, g.col).find_one(window=8)
        assert f.omega == om and oracle.is_clique(*g.numpy(), f.cliques[0])


@pytest.mark.parametrize("kind", ["thr", "tile"])
@pytest.mark.parametrize("min_w", [4, 8, 16, 99])
@pytest.mark.parametrize("key", ["ER400d", "ER150d", "RMAT13", "RMAT15", "K257", "K130", "T(36,12)", "CP8+K600",
                                 "CP12+K300", "planted", "Paley17", "ER700w8", "ER1000w8"])
def test_smem_expand_widths(key, min_w, kind, monkeypatch):
    """The shared-memory count pass (root matrix staged per block, entries
    grouped by slot; thread per candidate = expand_thr, tile per candidate =
    expand_smem) from width min_w up, against the oracle; 99 = off
    (global-memory tile / thread kernels)."""
    if min_w == 99 and kind == "tile":
        pytest.skip("same as kind=thr with the shared-memory pass off")
    monkeypatch.setenv("MCE_SMEM_KIND", kind)
    monkeypatch.setenv("MCE_SMEM_MIN_W", str(min_w))
    monkeypatch.setenv("MCE_SMEM_MIN_N", "1")  # every level of the width, however small
    monkeypatch.setenv("MCE_SMEM_PER_ROOT", "0")
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    # small budgets: the fused pass overflows and the (global-memory) write pass
    # must reproduce exactly the children the shared-memory count pass counted
    for kw in (dict(), dict(fused_levels=False), dict(clique_shortcut=False), dict(bound="size", heuristic="none"),
               # (with no heuristic RMAT15's chunked subtrees nest ~50 levels deep: 6 MB ran out
               # for 2 in 50 asynchronous k-core peel orders, 8 MB for 1 in ~600 -- a clean
               # MCE_ERR_BUDGET; the deterministic order makes the frontier sizes repeatable)
               dict(budget_bytes=8 << 20, heuristic="none", fused_levels=False, orientation="degeneracy_det"),
               dict(budget_bytes=24 << 20, heuristic="single_degree")):
        if kw.get("bound") == "size" and key in ("RMAT15", "RMAT13", "CP8+K600", "CP12+K300", "K257", "ER400d",
                                                 "ER700w8", "ER1000w8"):
            continue
        if "budget_bytes" in kw and (key.startswith("K") or key.startswith("CP")):
            continue  # 256-level chains: a 6 MB budget is below one candidate's chunk share (MCE_ERR_BUDGET)
        r = run_enum(g, **kw)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl), kw
    r = run_enum(g, smem_expand=False)
    assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl)
    f = mce().Graph(g.rowptr, g.col).find_one(window=4)
    assert f.omega == om and oracle.is_clique(*g.numpy(), f.cliques[0])


GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def golden(name):
    path = os.path.join(GOLDEN, f"{name}.json")
    if not os.path.exists(path):
        pytest.skip(f"{path} not written yet (scripts/make_golden_rmat.py)")
    with open(path) as f:
        return json.load(f)


def rmat_graph(name, device):
    if name in ("rmat22", "rmat26"):
        return G.make_config(name, device=device)
    if name.startswith("rmat26s"):  # configs[4]'s recipe (50 planted 20-cliques) at a smaller scale
        return G.make_config("rmat26", device=device, scale_override=int(name[7:]))
    return G.rmat(int(name[4:]), 16, 0.57, 0.19, 0.19, seed=1, device=device)


def check_stored_rows(rows, omega, rp, col, sample=64):
    """Every stored row: omega distinct ascending vertices, rows distinct and in
    lexicographic order; a spread sample is checked to be a clique."""
    assert rows.ndim == 2 and rows.shape[1] == omega
    assert np.all(np.diff(rows, axis=1) > 0)
    if rows.shape[0] > 1:
        order = np.lexsort(rows.T[::-1])
        assert np.array_equal(order, np.arange(rows.shape[0]))
        assert np.all(np.any(rows[1:] != rows[:-1], axis=1))
    for i in np.linspace(0, rows.shape[0] - 1, min(sample, rows.shape[0])).astype(np.int64):
        assert oracle.is_clique(rp, col, rows[i])


@pytest.mark.slow
@pytest.mark.parametrize("name", ["rmat20", "rmat22", "rmat26s20"])
def test_config_rmat_golden(name):
    """BASELINE configs[2] (rmat22) and the same recipe at scale 20: omega and
    the exact multiplicity against the oracle's count (tests/golden, written by
    scripts/make_golden_rmat.py from oracle/ only); the 2^16 stored rows are
    valid, distinct maximum cliques."""
    gd = golden(name)
    g = rmat_graph(name, "cuda")
    r = run_enum(g, max_cliques=1 << 16)
    assert (r.omega, r.count) == (gd["omega"], gd["multiplicity"])
    assert r.cliques.shape[0] == min(1 << 16, gd["multiplicity"])
    rp, col = g.rowptr.cpu().numpy(), g.col.cpu().numpy()
    check_stored_rows(r.cliques, r.omega, rp, col)


@pytest.mark.slow
@pytest.mark.parametrize("depth", [0, 3])
def test_config_rmat22_shards(depth):
    """configs[2] at "2 GPUs": two graph handles (two processes' state), the
    deterministic orientation computed by each, root (depth 0) or level-3 hash
    deal: the shards' multiplicities add up to the oracle's."""
    gd = golden("rmat22")
    g = rmat_graph("rmat22", "cuda")
    m = mce()
    parts = []
    for rank in range(2):
        h = m.Graph(g.rowptr, g.col)
        parts.append(h.enumerate(orientation="degeneracy_det", shard_rank=rank, shard_count=2, shard_depth=depth,
                                 max_cliques=1 << 10))
        h.close()
    omega = max(p.omega for p in parts)
    assert omega == gd["omega"]
    assert sum(p.count for p in parts if p.omega == omega) == gd["multiplicity"]


@pytest.mark.slow
def test_config_rmat26_golden():
    """BASELINE configs[4] on one GPU against the oracle's count (when the
    oracle run has been committed)."""
    gd = golden("rmat26")
    g = rmat_graph("rmat26", "cuda")
    r = run_enum(g, max_cliques=1 << 12)
    assert (r.omega, r.count) == (gd["omega"], gd["multiplicity"])
    check_stored_rows(r.cliques, r.omega, g.rowptr.cpu().numpy(), g.col.cpu().numpy(), sample=16)


@pytest.mark.parametrize("min_w", [1, 2, 8])
@pytest.mark.parametrize("key", ["ER400d", "RMAT13", "RMAT15", "K130", "K257", "T(36,12)", "CP8+K600", "CP12+K300",
                                 "planted", "ER700w8", "er2000", "BA5k"])
def test_reroot(key, min_w, monkeypatch):
    """Re-rooted candidates (every level >= 2 of at least min_w words becomes a
    set of roots over the candidates' own sets, nested level after level with
    min_w = 1): same answer as the oracle, with and without completions, and
    under a small budget (chunked levels), and find-one."""
    monkeypatch.setenv("MCE_REROOT_MIN_W", str(min_w))
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    for kw in (dict(), dict(clique_shortcut=False), dict(fused_levels=False), dict(smem_expand=False),
               dict(budget_bytes=24 << 20, heuristic="single_degree")):
        if "budget_bytes" in kw and (key.startswith("K") or key.startswith("CP") or min_w == 1):
            continue  # (nested re-rooting on every level holds every level's derived arrays)
        r = run_enum(g, **kw)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl), kw
    f = mce().Graph(g.rowptr, g.col).find_one(window=4)
    assert f.omega == om and oracle.is_clique(*g.numpy(), f.cliques[0])


@pytest.mark.parametrize("g", ["16", "8", "32"])
@pytest.mark.parametrize("key", ["ER400d", "RMAT13", "RMAT15", "K130", "K257", "T(36,12)", "CP8+K600", "CP12+K300",
                                 "planted", "ER700w8", "Paley17"])
def test_wide_lockstep(key, g, monkeypatch):
    """The wide count pass (expand_wide: global rows, lockstep G-lane tiles with
    W / G words per lane, order stored from colour need - k up) forced onto
    every level of 4 words or more (shared-memory pass off), against the oracle."""
    monkeypatch.setenv("MCE_WIDE_MIN_W", "4")
    monkeypatch.setenv("MCE_WIDE_G", g)
    monkeypatch.setenv("MCE_SMEM_MIN_W", "99")
    g_ = GRAPHS[key]()
    om, cl = oracle_answer(key)
    for kw in (dict(), dict(clique_shortcut=False), dict(fused_levels=False), dict(reroot=False),
               dict(budget_bytes=24 << 20, heuristic="single_degree"), dict(bound="size", heuristic="none")):
        if "budget_bytes" in kw and (key.startswith("K") or key.startswith("CP")):
            continue
        if kw.get("bound") == "size" and key in ("RMAT15", "RMAT13", "CP8+K600", "CP12+K300", "K257", "ER400d",
                                                 "ER700w8"):
            continue
        r = run_enum(g_, **kw)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl), kw
    f = mce().Graph(g_.rowptr, g_.col).find_one(window=4)
    assert f.omega == om and oracle.is_clique(*g_.numpy(), f.cliques[0])


@pytest.mark.parametrize("key", ["RMAT15", "RMAT13", "CP8+K600", "CP12+K300", "K130", "ER400d", "ER700w8", "planted",
                                 "T(36,12)", "Paley17", "BA5k", "er2000"])
def test_root_colour_filter(key, monkeypatch):
    """Root colour filter (colour.cu, reading 14) forced on at every size (MCE_ROOT_COLOUR_MIN_S=1):
    the greedy colouring of the vertices of core >= need - 1 and the per-root colour bound drop roots, never a
    maximum clique; enumeration (several heuristics: different need) and find-one against the oracle, and the
    filter off gives the same answer."""
    monkeypatch.setenv("MCE_ROOT_COLOUR_MIN_S", "1")
    g = GRAPHS[key]()
    om, cl = oracle_answer(key)
    for kw in (dict(), dict(heuristic="single_degree"), dict(heuristic="none"), dict(root_colour=False),
               dict(orientation="degeneracy_det")):
        if kw.get("heuristic") == "none" and key not in ("RMAT13", "planted", "BA5k", "er2000", "ER400d"):
            continue  # (no bound: exponential on the dense and hub-core graphs)
        r = run_enum(g, **kw)
        assert (r.omega, r.count) == (om, len(cl)) and np.array_equal(r.cliques, cl), kw
    m = mce()
    gg = m.Graph(g.rowptr, g.col)
    r = gg.find_one(window=4)
    assert r.omega == om and oracle.is_clique(*g.numpy(), r.cliques[0])
