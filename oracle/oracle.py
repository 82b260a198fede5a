"""ctypes wrapper around mce_oracle.c (plain C, fp-free, single-threaded).

TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py.
"""

from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mce_oracle.c")
_LIB = os.path.join(_HERE, "libmce_oracle.so")
_lib = None

_i64p = ctypes.POINTER(ctypes.c_int64)
_i32p = ctypes.POINTER(ctypes.c_int32)


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (the checker is built, not used, by build())."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_core_numbers.restype = ctypes.c_int32
        lib.oracle_core_numbers.argtypes = [ctypes.c_int64, _i64p, _i32p, _i32p, _i32p]
        lib.oracle_greedy.restype = ctypes.c_int32
        lib.oracle_greedy.argtypes = [ctypes.c_int64, _i64p, _i32p, _i64p, ctypes.c_int64, _i32p, _i32p]
        lib.oracle_mce.restype = ctypes.c_int64
        lib.oracle_mce.argtypes = [ctypes.c_int64, _i64p, _i32p, ctypes.c_int32, ctypes.c_int32, _i32p]
        lib.oracle_mce_ex.restype = ctypes.c_int64
        lib.oracle_mce_ex.argtypes = [ctypes.c_int64, _i64p, _i32p, ctypes.c_int32, ctypes.c_int32,
                                      ctypes.c_int32, _i32p]
        lib.oracle_mce_plain.restype = ctypes.c_int64
        lib.oracle_mce_plain.argtypes = [ctypes.c_int64, _i64p, _i32p, ctypes.c_int32, ctypes.c_int32,
                                         ctypes.c_int32, _i32p]
        lib.oracle_mce_fetch.restype = None
        lib.oracle_mce_fetch.argtypes = [_i32p]
        lib.oracle_kclique_counts.restype = ctypes.c_int32
        lib.oracle_kclique_counts.argtypes = [ctypes.c_int64, _i64p, _i32p, ctypes.c_int32, _i64p]
        lib.oracle_is_clique.restype = ctypes.c_int32
        lib.oracle_is_clique.argtypes = [_i64p, _i32p, _i32p, ctypes.c_int32]
        _lib = lib
    return _lib


def _csr(rowptr, col):
    rowptr = np.ascontiguousarray(np.asarray(rowptr, dtype=np.int64))
    col = np.ascontiguousarray(np.asarray(col, dtype=np.int32))
    return rowptr, col


def _p64(a):
    return a.ctypes.data_as(_i64p)


def _p32(a):
    return a.ctypes.data_as(_i32p)


def core_numbers(rowptr, col) -> Tuple[np.ndarray, np.ndarray, int]:
    """(core number per vertex, Batagelj-Zaversnik peel order, degeneracy)."""
    rowptr, col = _csr(rowptr, col)
    n = rowptr.size - 1
    core = np.zeros(n, dtype=np.int32)
    order = np.zeros(n, dtype=np.int32)
    d = _load().oracle_core_numbers(n, _p64(rowptr), _p32(col), _p32(core), _p32(order))
    return core, order, int(d)


def greedy(rowptr, col, threshold, h: int) -> Tuple[int, np.ndarray, np.ndarray]:
    """Multi-run greedy heuristic (Algorithm 1).  Returns (omega_bar, run sizes, best clique)."""
    rowptr, col = _csr(rowptr, col)
    n = rowptr.size - 1
    thr = np.ascontiguousarray(np.asarray(threshold, dtype=np.int64))
    h = max(0, min(int(h), n))
    runs = np.zeros(max(h, 1), dtype=np.int32)
    maxdeg = int(np.diff(rowptr).max()) if n else 0
    best = np.zeros(maxdeg + 2, dtype=np.int32)
    w = _load().oracle_greedy(n, _p64(rowptr), _p32(col), _p64(thr), h, _p32(runs), _p32(best))
    return int(w), runs[:h], best[:w]


def max_cliques(rowptr, col, lb: int = 0, bound: str = "color", tight: bool = False) -> Tuple[int, np.ndarray]:
    """(omega, all maximum cliques as a sorted int32 [count, omega] array).

    bound: "size" = |C|+|P| (PAPER.md II-B-3 first option), "color" = greedy
    colouring bound (II-B-3 "tighter upper bound ... vertex coloring"), both
    on oracle_mce's degeneracy-ordered bitset search; "plain" = oracle_mce_plain,
    the literal list-based II-A search with the |C|+|P| bound over the
    paper's degree orientation (IV-C, line 131), "plain_id" the same in
    vertex-id order (no k-core, no bitsets, no colouring: independent of
    both the other oracle and the CUDA path's layout).
    """
    rowptr, col = _csr(rowptr, col)
    n = rowptr.size - 1
    lib = _load()
    om = ctypes.c_int32(0)
    if bound in ("plain", "plain_id"):
        cnt = lib.oracle_mce_plain(n, _p64(rowptr), _p32(col), int(lb), int(bound == "plain"), 0,
                                   ctypes.byref(om))
    else:
        b = {"size": 0, "color": 1}[bound]
        cnt = lib.oracle_mce_ex(n, _p64(rowptr), _p32(col), int(lb), b, 2 * int(tight), ctypes.byref(om))
    if cnt < 0:
        raise ValueError("oracle: a vertex has more than 65536 later neighbours")
    omega = int(om.value)
    out = np.zeros((cnt, omega), dtype=np.int32)
    lib.oracle_mce_fetch(_p32(out) if out.size else None)
    return omega, out


def count_max_cliques(rowptr, col, lb: int = 0, bound: str = "color", tight: bool = False) -> Tuple[int, int]:
    """(omega, multiplicity) without storing the cliques (count-only mode).

    Same searches as max_cliques; for graphs whose maximum cliques do not fit
    in host memory (R-MAT scale 22: 3 * 2^26 cliques of 223 vertices).
    tight (colour / size bounds only): stop at a node where |C| + |P| equals
    the size sought and test P for being a clique (mce_oracle.c expand()).
    """
    rowptr, col = _csr(rowptr, col)
    n = rowptr.size - 1
    lib = _load()
    om = ctypes.c_int32(0)
    if bound in ("plain", "plain_id"):
        cnt = lib.oracle_mce_plain(n, _p64(rowptr), _p32(col), int(lb), int(bound == "plain"), 1,
                                   ctypes.byref(om))
    else:
        b = {"size": 0, "color": 1}[bound]
        cnt = lib.oracle_mce_ex(n, _p64(rowptr), _p32(col), int(lb), b, 1 | (2 * int(tight)), ctypes.byref(om))
    if cnt < 0:
        raise ValueError("oracle: a vertex has more than 65536 later neighbours")
    return int(om.value), int(cnt)


def kclique_counts(rowptr, col, kmax: int) -> np.ndarray:
    """counts[k-1] = number of k-cliques, k = 1..kmax."""
    rowptr, col = _csr(rowptr, col)
    n = rowptr.size - 1
    counts = np.zeros(max(kmax, 1), dtype=np.int64)
    _load().oracle_kclique_counts(n, _p64(rowptr), _p32(col), int(kmax), _p64(counts))
    return counts[:kmax]


def is_clique(rowptr, col, verts) -> bool:
    rowptr, col = _csr(rowptr, col)
    v = np.ascontiguousarray(np.asarray(verts, dtype=np.int32))
    return bool(_load().oracle_is_clique(_p64(rowptr), _p32(col), _p32(v), int(v.size)))


def default_threshold(rowptr, col, kind: str) -> np.ndarray:
    """Threshold used by the greedy heuristic: 'degree' or 'core' (IV-A)."""
    rowptr, col = _csr(rowptr, col)
    if kind == "degree":
        return np.diff(rowptr).astype(np.int64)
    if kind == "core":
        return core_numbers(rowptr, col)[0].astype(np.int64)
    raise ValueError(kind)
