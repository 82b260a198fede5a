"""Seeded synthetic graphs (CSR) for the maximum-clique workloads.

Shapes follow the workloads named in BASELINE.json `configs` (sparse
Erdos-Renyi with a planted clique, Barabasi-Albert, R-MAT power-law graphs,
dense G(n, 1/2)) and the paper's preprocessing of its inputs (PAPER.md
Sec. V: graphs made undirected, loop-free, vertex indices
randomised).  Closed-form graphs (K_n, C_n, Turan T(n,k), Paley P(q)) are the
test pins of DESIGN.md.

Randomness is a counter-based generator (SplitMix64 over (seed, stream,
index)), implemented on torch int64 tensors, so a graph is bit-identical
whether it is built on the CPU or on a CUDA device.  Nothing here computes
cliques, cores or heuristics.
"""

from __future__ import annotations

import dataclasses
from typing import List, Optional, Sequence

import numpy as np
import torch

_M64 = (1 << 64) - 1


def _s64(x: int) -> int:
    """Reinterpret an unsigned 64-bit Python int as signed int64."""
    x &= _M64
    return x - (1 << 64) if x >= (1 << 63) else x


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_C1 = _s64(0xBF58476D1CE4E5B9)
_C2 = _s64(0x94D049BB133111EB)


def _srl(z: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift on int64 tensors."""
    return (z >> s) & ((1 << (64 - s)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """SplitMix64 output function on int64 tensors (wrapping arithmetic)."""
    z = x + _GOLDEN
    z = (z ^ _srl(z, 30)) * _C1
    z = (z ^ _srl(z, 27)) * _C2
    return z ^ _srl(z, 31)


def splitmix64_py(x: int) -> int:
    """Pure-Python SplitMix64 (the pin for the tensor version)."""
    z = (x + 0x9E3779B97F4A7C15) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def _stream_base(seed: int, stream: int) -> int:
    return _s64(splitmix64_py((seed * 0x100000001B3 + stream * 0x9E3779B1) & _M64))


def rand_u64(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """64 random bits for each counter in `idx` (int64 tensor)."""
    return splitmix64(idx * _GOLDEN + _stream_base(seed, stream))


def rand_uniform(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """float64 uniform in [0, 1) with 53 random bits per counter."""
    return _srl(rand_u64(seed, stream, idx), 11).to(torch.float64) * (2.0 ** -53)


@dataclasses.dataclass
class Graph:
    """Undirected simple graph in CSR (both directions stored, lists sorted)."""

    n: int
    rowptr: torch.Tensor  # int64 [n+1]
    col: torch.Tensor  # int32 [nnz], nnz = 2|E|
    name: str = ""
    planted: Optional[List[List[int]]] = None

    @property
    def num_edges(self) -> int:
        return int(self.col.numel()) // 2

    def to(self, device) -> "Graph":
        return dataclasses.replace(self, rowptr=self.rowptr.to(device), col=self.col.to(device))

    def numpy(self):
        return self.rowptr.cpu().numpy(), self.col.cpu().numpy()

    def edges(self) -> np.ndarray:
        """Undirected edge list (u < v) as an int64 [|E|, 2] array."""
        rp, col = self.numpy()
        src = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(rp))
        m = src < col
        return np.stack([src[m], col[m].astype(np.int64)], axis=1)


def _csr_from_keys(n: int, key: torch.Tensor, name: str = "") -> Graph:
    """CSR (both directions, rows ascending) from sorted unique keys a * n + b, a < b.

    Row v is [a < v : (a, v) an edge] ++ [b > v : (v, b) an edge]: the upper
    half comes grouped by a and sorted by b with the keys; the lower half is
    one more sort of b * n + a.  Every part is ascending and the lower part is
    below v, so the concatenation is the sorted row.  Memory stays a few
    copies of |E| (R-MAT scale 26: 10^9 edges on one GPU).
    """
    device = key.device
    m = key.numel()
    a = (key // n).to(torch.int32)
    b = (key - a.to(torch.int64) * n).to(torch.int32)
    up = torch.bincount(a, minlength=n) if m else torch.zeros(n, dtype=torch.int64, device=device)
    lo = torch.bincount(b, minlength=n) if m else torch.zeros(n, dtype=torch.int64, device=device)
    rowptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    rowptr[1:] = torch.cumsum(up + lo, 0)
    col = torch.empty(2 * m, dtype=torch.int32, device=device)
    if m:
        # upper half, in key order: rank of each entry inside its row group a
        ustart = torch.cumsum(up, 0) - up
        idx = torch.arange(m, dtype=torch.int64, device=device)
        al = a.to(torch.int64)
        col[rowptr[:-1][al] + lo[al] + (idx - ustart[al])] = b
        del al, ustart
        # lower half, sorted by (b, a)
        k2, _ = torch.sort(b.to(torch.int64) * n + a.to(torch.int64))
        del a, b
        b2 = k2 // n
        a2 = (k2 - b2 * n).to(torch.int32)
        del k2
        lstart = torch.cumsum(lo, 0) - lo
        col[rowptr[:-1][b2] + (idx - lstart[b2])] = a2
        del b2, a2, idx, lstart
    return Graph(n=n, rowptr=rowptr, col=col, name=name)


def edge_keys(n: int, src: torch.Tensor, dst: torch.Tensor) -> torch.Tensor:
    """Undirected keys min * n + max of the non-loop pairs (unsorted, with duplicates)."""
    src = src.to(torch.int64)
    dst = dst.to(torch.int64)
    keep = src != dst
    src, dst = src[keep], dst[keep]
    return torch.minimum(src, dst) * n + torch.maximum(src, dst)


def from_keys(n: int, keys: torch.Tensor, name: str = "") -> Graph:
    """Graph from undirected keys (duplicates allowed)."""
    return _csr_from_keys(n, torch.unique(keys), name=name)


def from_edges(n: int, src: torch.Tensor, dst: torch.Tensor, name: str = "") -> Graph:
    """Symmetrise, drop self loops and duplicates, build sorted CSR."""
    return from_keys(n, edge_keys(n, src, dst), name=name)


def _pairs_from_mask(n: int, keep_fn, device, chunk_rows: int = 256):
    """Enumerate pairs i<j row-chunk by row-chunk, keeping those keep_fn accepts."""
    srcs, dsts = [], []
    j = torch.arange(n, dtype=torch.int64, device=device)
    for r0 in range(0, n, chunk_rows):
        i = torch.arange(r0, min(n, r0 + chunk_rows), dtype=torch.int64, device=device)
        ii = i[:, None].expand(-1, n)
        jj = j[None, :].expand(i.numel(), -1)
        upper = jj > ii
        mask = upper & keep_fn(ii, jj)
        srcs.append(ii[mask])
        dsts.append(jj[mask])
    return torch.cat(srcs), torch.cat(dsts)


# ---------------------------------------------------------------------------
# Closed-form graphs (test pins)
# ---------------------------------------------------------------------------


def complete_graph(n: int, device="cpu") -> Graph:
    s, d = _pairs_from_mask(n, lambda i, j: torch.ones_like(i, dtype=torch.bool), device)
    return from_edges(n, s, d, name=f"K{n}")


def cycle_graph(n: int, device="cpu") -> Graph:
    i = torch.arange(n, dtype=torch.int64, device=device)
    return from_edges(n, i, (i + 1) % n, name=f"C{n}")


def turan_graph(n: int, k: int, device="cpu") -> Graph:
    """Complete k-partite graph with parts as equal as possible (part = v mod k)."""
    s, d = _pairs_from_mask(n, lambda i, j: (i % k) != (j % k), device)
    return from_edges(n, s, d, name=f"T({n},{k})")


def paley_graph(q: int, device="cpu") -> Graph:
    """Paley graph on GF(q), q prime and q = 1 (mod 4)."""
    squares = torch.zeros(q, dtype=torch.bool, device=device)
    x = torch.arange(1, q, dtype=torch.int64, device=device)
    squares[(x * x) % q] = True
    s, d = _pairs_from_mask(q, lambda i, j: squares[(j - i) % q], device)
    return from_edges(q, s, d, name=f"Paley({q})")


# ---------------------------------------------------------------------------
# Random graphs (workload shapes)
# ---------------------------------------------------------------------------

_STREAM_ER = 11
_STREAM_PERM = 12
_STREAM_PLANT = 13
_STREAM_BA = 14
_STREAM_RMAT = 100  # + level


def erdos_renyi(n: int, p: float, seed: int, device="cpu") -> Graph:
    """G(n, p): pair (i<j) is an edge iff U(seed, i*n+j) < p."""

    def keep(ii, jj):
        return rand_uniform(seed, _STREAM_ER, ii * n + jj) < p

    s, d = _pairs_from_mask(n, keep, device)
    return from_edges(n, s, d, name=f"G({n},{p})s{seed}")


def planted_clique_edges(n: int, count: int, size: int, seed: int, device="cpu"):
    """`count` vertex-disjoint cliques of `size` random vertices: (src, dst, chosen rows)."""
    if count * size > n:
        raise ValueError("not enough vertices to plant the cliques")
    keys = rand_u64(seed, _STREAM_PLANT, torch.arange(n, dtype=torch.int64, device=device))
    chosen = torch.argsort(keys)[: count * size].reshape(count, size)
    del keys
    chosen, _ = torch.sort(chosen, dim=1)
    ii, jj = torch.triu_indices(size, size, offset=1, device=device)
    return chosen[:, ii].reshape(-1), chosen[:, jj].reshape(-1), chosen


def plant_cliques(g: Graph, count: int, size: int, seed: int) -> Graph:
    """Add `count` vertex-disjoint cliques of `size` vertices chosen at random."""
    n = g.n
    device = g.rowptr.device
    add_s, add_d, chosen = planted_clique_edges(n, count, size, seed, device)
    rp = g.rowptr
    src = torch.repeat_interleave(torch.arange(n, dtype=torch.int64, device=device), rp[1:] - rp[:-1])
    up = src < g.col
    keys = torch.cat([src[up] * n + g.col[up].to(torch.int64), edge_keys(n, add_s, add_d)])
    del src, up
    out = from_keys(n, keys, name=f"{g.name}+{count}x K{size}")
    out.planted = (g.planted or []) + chosen.cpu().tolist()
    return out


def cocktail_party_join(j: int, t: int, seed: int) -> Graph:
    """Cocktail-party graph CP(j) (K_2j minus a perfect matching) joined with K_t,
    vertex ids permuted with a seeded permutation.  Closed form (test pin):
    omega = j + t with 2^j maximum cliques (one vertex of every non-adjacent
    pair), the structure of the R-MAT hub core."""
    n = 2 * j + t
    u, v = np.triu_indices(n, 1)
    keep = ~((u < 2 * j) & (v < 2 * j) & (u // 2 == v // 2))
    perm = torch.argsort(rand_u64(seed, 7, torch.arange(n, dtype=torch.int64))).numpy()
    return from_edges(n, torch.from_numpy(perm[u[keep]].astype(np.int64)),
                      torch.from_numpy(perm[v[keep]].astype(np.int64)), name=f"CP({j})+K{t}")


def barabasi_albert(n: int, m: int, seed: int) -> Graph:
    """Barabasi-Albert preferential attachment (networkx-style, sequential).

    Vertices 0..m-1 start isolated; vertex m attaches to all of them; every
    later vertex attaches to m distinct targets drawn uniformly from the list
    of edge endpoints so far (degree-proportional).  Draw t uses counter t.
    """
    if n <= m:
        return from_edges(n, torch.zeros(0, dtype=torch.int64), torch.zeros(0, dtype=torch.int64), name="BA")
    total_draws_est = (n - m) * m * 2 + 1024
    draws = rand_uniform(seed, _STREAM_BA, torch.arange(total_draws_est, dtype=torch.int64)).numpy()
    rep = np.empty(2 * m * (n - m), dtype=np.int64)  # repeated endpoints
    src = np.empty((n - m) * m, dtype=np.int64)
    dst = np.empty((n - m) * m, dtype=np.int64)
    rep_len = 0
    e = 0
    t = 0
    targets = list(range(m))
    for v in range(m, n):
        for u in targets:
            src[e] = v
            dst[e] = u
            e += 1
        rep[rep_len : rep_len + m] = targets
        rep[rep_len + m : rep_len + 2 * m] = v
        rep_len += 2 * m
        if v + 1 == n:
            break
        chosen = set()
        tl = []
        while len(tl) < m:
            if t >= total_draws_est:
                extra = rand_uniform(seed, _STREAM_BA, torch.arange(t, t + 1 << 16, dtype=torch.int64)).numpy()
                draws = np.concatenate([draws, extra])
                total_draws_est = draws.size
            x = int(rep[int(draws[t] * rep_len)])
            t += 1
            if x not in chosen:
                chosen.add(x)
                tl.append(x)
        targets = tl
    return from_edges(n, torch.from_numpy(src[:e]), torch.from_numpy(dst[:e]), name=f"BA({n},{m})s{seed}")


def rmat(scale: int, edge_factor: int, a: float, b: float, c: float, seed: int,
         device="cpu", permute: bool = True, chunk: int = 1 << 24, plant=None) -> Graph:
    """R-MAT (Chakrabarti et al.) with 2^scale vertices and edge_factor*2^scale draws.

    Each draw descends `scale` levels picking quadrant (0,0),(0,1),(1,0),(1,1)
    with probabilities a, b, c, 1-a-b-c.  Vertex ids are then randomly
    permuted (the paper randomises indices).  `plant` =
    (count, size, seed) adds planted cliques exactly as plant_cliques does,
    without building the graph twice.
    """
    n = 1 << scale
    m = edge_factor * n
    ab = a + b
    abc = a + b + c
    label = None
    if permute:
        keys = rand_u64(seed, _STREAM_PERM, torch.arange(n, dtype=torch.int64, device=device))
        order = torch.argsort(keys)
        label = torch.empty_like(order)
        label[order] = torch.arange(n, dtype=torch.int64, device=device)
        del keys, order
    parts = []
    for e0 in range(0, m, chunk):
        e = torch.arange(e0, min(m, e0 + chunk), dtype=torch.int64, device=device)
        s = torch.zeros_like(e)
        d = torch.zeros_like(e)
        for lvl in range(scale):
            u = rand_uniform(seed, _STREAM_RMAT + lvl, e)
            sb = (u >= ab).to(torch.int64)
            db = ((u >= a) & (u < ab)) | (u >= abc)
            bit = 1 << (scale - 1 - lvl)
            s += sb * bit
            d += db.to(torch.int64) * bit
            del u, sb, db
        if label is not None:
            s = label[s]
            d = label[d]
        parts.append(edge_keys(n, s, d))
        del e, s, d
    del label
    chosen = None
    if plant is not None:
        ps, pd, chosen = planted_clique_edges(n, plant[0], plant[1], plant[2], device)
        parts.append(edge_keys(n, ps, pd))
    keys = torch.cat(parts)
    del parts
    name = f"RMAT{scale}ef{edge_factor}s{seed}"
    if plant is not None:
        name += f"+{plant[0]}x K{plant[1]}"
    g = from_keys(n, keys, name=name)
    if chosen is not None:
        g.planted = chosen.cpu().tolist()
    return g


# ---------------------------------------------------------------------------
# The BASELINE.json workloads
# ---------------------------------------------------------------------------

CONFIGS = {
    # configs[0]: small case the oracle finishes in seconds
    "er2000": dict(desc="Erdos-Renyi G(n=2000, p=0.005) seed 1 with a planted 12-clique"),
    # configs[1]: the headline 1-GPU workload
    "ba1m": dict(desc="Barabasi-Albert n=1M, m=4"),
    # configs[2]: strong-scaling workload at 1/2/4/8 GPUs
    "rmat22": dict(desc="R-MAT scale 22, edge factor 16 (a=0.57, b=c=0.19)"),
    # configs[3]: dense, windowed single-maximum-clique search
    "dense800": dict(desc="G(n=800, p=0.5), windowed find-one"),
    # configs[4]: 8-GPU workload
    "rmat26": dict(desc="R-MAT scale 26, edge factor 16 with 50 planted 20-cliques"),
}


def make_config(name: str, device="cpu", scale_override: Optional[int] = None) -> Graph:
    """Build one of the BASELINE.json workloads (optionally at a smaller R-MAT scale)."""
    if name == "er2000":
        g = erdos_renyi(2000, 0.005, seed=1, device=device)
        return plant_cliques(g, 1, 12, seed=1)
    if name == "ba1m":
        return barabasi_albert(1_000_000, 4, seed=1).to(device)
    if name == "rmat22":
        return rmat(scale_override or 22, 16, 0.57, 0.19, 0.19, seed=1, device=device)
    if name == "dense800":
        return erdos_renyi(800, 0.5, seed=1, device=device)
    if name == "rmat26":
        return rmat(scale_override or 26, 16, 0.57, 0.19, 0.19, seed=1, device=device, plant=(50, 20, 1))
    raise KeyError(name)


def degree_stats(g: Graph) -> dict:
    deg = (g.rowptr[1:] - g.rowptr[:-1]).to(torch.float64)
    return dict(n=g.n, m=g.num_edges, avg_deg=float(deg.mean()) if g.n else 0.0,
                max_deg=int(deg.max()) if g.n else 0)
