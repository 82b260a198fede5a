"""Brute-force subset enumeration for tiny graphs (n <= 20) -- an oracle pin.

Independent of oracle/ (no shared code): every vertex subset S is a bitmask;
clique[S] is computed by the recurrence clique[S] = clique[S - {j}] and
(S - {j}) is contained in N(j), j = highest vertex of S.  This is the
definition of a clique (PAPER.md II line 47) checked for all 2^n subsets.
"""

from __future__ import annotations

import itertools
from typing import List, Tuple

import numpy as np


def adjacency_masks(n: int, edges) -> np.ndarray:
    adj = np.zeros(n, dtype=np.int64)
    for u, v in edges:
        adj[u] |= 1 << int(v)
        adj[v] |= 1 << int(u)
    return adj


def all_clique_flags(n: int, edges) -> np.ndarray:
    """clique[mask] for every mask in [0, 2^n)."""
    assert n <= 22
    adj = adjacency_masks(n, edges)
    clique = np.zeros(1 << n, dtype=bool)
    clique[0] = True
    for j in range(n):
        lo = np.arange(1 << j, dtype=np.int64)  # masks of vertices < j
        clique[(1 << j) + lo] = clique[lo] & ((lo & adj[j]) == lo)
    return clique


def popcounts(n: int) -> np.ndarray:
    pc = np.zeros(1 << n, dtype=np.int64)
    for j in range(n):
        pc[1 << j: 1 << (j + 1)] = pc[: 1 << j] + 1
    return pc


def max_cliques(n: int, edges) -> Tuple[int, List[List[int]]]:
    if n == 0:
        return 0, [[]]
    flags = all_clique_flags(n, edges)
    pc = popcounts(n)
    omega = int(pc[flags].max())
    masks = np.nonzero(flags & (pc == omega))[0]
    cl = sorted([[v for v in range(n) if (int(m) >> v) & 1] for m in masks])
    return omega, cl


def kclique_counts(n: int, edges, kmax: int) -> List[int]:
    flags = all_clique_flags(n, edges)
    pc = popcounts(n)
    return [int(np.count_nonzero(flags & (pc == k))) for k in range(1, kmax + 1)]


def core_numbers_by_definition(n: int, edges) -> List[int]:
    """core(v) = max k such that v is in the k-core, the k-core being what is
    left after repeatedly deleting vertices of degree < k (Seidman 1983,
    PAPER.md II-B-2 line 61)."""
    nbrs = [set() for _ in range(n)]
    for u, v in edges:
        nbrs[u].add(v)
        nbrs[v].add(u)
    core = [0] * n
    for k in itertools.count(1):
        alive = set(range(n))
        changed = True
        while changed:
            changed = False
            for v in list(alive):
                if len(nbrs[v] & alive) < k:
                    alive.discard(v)
                    changed = True
        if not alive:
            break
        for v in alive:
            core[v] = k
    return core
