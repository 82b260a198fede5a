"""Python API over the C ABI (argument marshalling only; all compute on the GPU).

    g = Graph(rowptr, col)              # mce_load_csr  (torch/numpy, host or CUDA)
    r = g.enumerate()                   # mce_enumerate: omega, multiplicity, all maximum cliques
    r = g.find_one(window=1024)         # mce_find_one:  windowed single-maximum-clique search
    core, order, d = g.preprocess()     # k-core numbers + orientation order
    wbar, clique, runs = g.heuristic("multi_degree")

PAPER.md II line 47 states the problem; IV-A..IV-E the method (see
include/mce.h for every call's contract).
"""

from __future__ import annotations

import ctypes
import os
import dataclasses
from typing import Callable, List, Optional

import numpy as np

from . import _lib
from ._lib import BOUND, BOUND_SYNC, HEURISTIC, ORIENT, Options, check, lib

try:  # torch is plumbing here: device memory and streams
    import torch
except ImportError:  # pragma: no cover
    torch = None


@dataclasses.dataclass
class Result:
    omega: int
    count: int  # multiplicity (exact, even when the stored list is truncated)
    cliques: np.ndarray  # int32 [stored, omega]: each row ascending, rows lexicographic
    truncated: bool
    levels: List[int]  # candidates expanded per |C| (index k = |C|)
    timing: dict


def _ptr_and_where(x, dtype):
    """(pointer, where, keepalive) for a torch tensor or a numpy array."""
    if torch is not None and isinstance(x, torch.Tensor):
        t = x.contiguous()
        want = {np.int64: torch.int64, np.int32: torch.int32}[dtype]
        if t.dtype != want:
            t = t.to(want)
        where = _lib.WHERE_DEVICE if t.is_cuda else _lib.WHERE_HOST
        return ctypes.c_void_p(t.data_ptr()), where, t
    a = np.ascontiguousarray(np.asarray(x, dtype=dtype))
    return a.ctypes.data_as(ctypes.c_void_p), _lib.WHERE_HOST, a


def _current_stream(device: int):
    if torch is not None and torch.cuda.is_available():
        return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)
    return None


def make_options(orientation="degeneracy", heuristic="multi_degree", heuristic_runs=0, bound="color",
                 lower_bound=0, window=0, budget_bytes=0, max_cliques=0, shard_rank=0, shard_count=1,
                 bound_sync: Optional[Callable[[int, int], tuple]] = None, verbose=0, legacy_roots=False,
                 fused_levels=True, clique_shortcut=True, fused_expand=True, overlap=True, shard_depth=0,
                 smem_expand=True, reroot=True, root_colour=True):
    o = Options()
    lib().mce_default_options(ctypes.byref(o))
    o.orientation = ORIENT[orientation]
    o.heuristic = HEURISTIC[heuristic]
    o.heuristic_runs = int(heuristic_runs)
    o.bound = BOUND[bound]
    o.lower_bound = int(lower_bound)
    o.window = int(window)
    o.budget_bytes = int(budget_bytes)
    o.max_cliques = int(max_cliques)
    o.shard_rank = int(shard_rank)
    o.shard_count = int(shard_count)
    o.verbose = int(verbose) or int(os.environ.get("MCE_VERBOSE", "0") or 0)
    o.legacy_roots = int(bool(legacy_roots))
    o.no_fused_levels = int(not fused_levels)
    o.no_clique_shortcut = int(not clique_shortcut)
    o.no_fused_expand = int(not fused_expand)
    o.no_overlap = int(not overlap)
    o.shard_depth = int(shard_depth)
    o.no_smem_expand = int(not smem_expand)
    o.no_reroot = int(not reroot)
    o.no_root_colour = int(not root_colour) or int(os.environ.get("MCE_NO_ROOT_COLOUR", "0") or 0)
    keep = None
    if bound_sync is not None:
        errors = []

        def _cb(local_best, local_active, gactive, _user):
            # an exception must not unwind through the C frames: report it with
            # the negative sentinel (the engine stops with MCE_ERR_SYNC) and
            # re-raise it from the Python call (SyncGuard)
            try:
                gb, ga = bound_sync(int(local_best), int(local_active))
                gactive[0] = int(ga)
                return max(int(gb), 0)
            except BaseException as e:  # noqa: BLE001
                errors.append(e)
                gactive[0] = 0
                return -1

        keep = _SyncGuard(BOUND_SYNC(_cb), errors)
        o.bound_sync = keep.fn
    return o, keep


class _SyncGuard:
    """Keeps the ctypes callback alive for the call and re-raises what it caught."""

    def __init__(self, fn, errors):
        self.fn = fn
        self.errors = errors

    def reraise(self):
        if self.errors:
            raise self.errors[0]


class Graph:
    """A graph resident on one GPU (mce_load_csr)."""

    def __init__(self, rowptr, col, device: int = 0, validate: bool = False, stream=None):
        rp, where_r, self._krp = _ptr_and_where(rowptr, np.int64)
        cp, where_c, self._kcol = _ptr_and_where(col, np.int32)
        if where_r != where_c:
            raise ValueError("rowptr and col must both be host or both be device memory")
        self.n = int(self._krp.shape[0]) - 1
        self.device = device
        self._stream = stream if stream is not None else _current_stream(device)
        h = ctypes.c_void_p()
        check(lib().mce_load_csr(device, self.n, rp, cp, where_r, int(validate), self._stream, ctypes.byref(h)))
        self._h = h
        self._krp = self._kcol = None  # the library holds its own device copy

    def close(self):
        if getattr(self, "_h", None):
            lib().mce_graph_free(self._h)
            self._h = None

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass

    def clear_cache(self):
        check(lib().mce_graph_clear_cache(self._h))

    def preprocess(self, orientation: str = "degeneracy"):
        core = np.zeros(max(self.n, 1), np.int32)
        order = np.zeros(max(self.n, 1), np.int32)
        d = ctypes.c_int32()
        check(lib().mce_preprocess(self._h, ORIENT[orientation], core.ctypes.data_as(ctypes.c_void_p),
                                   order.ctypes.data_as(ctypes.c_void_p), _lib.WHERE_HOST, ctypes.byref(d)))
        return core[: self.n], order[: self.n], int(d.value)

    def order_into(self, out, orientation: str = "degeneracy"):
        """Preprocess (cached) and copy the orientation order into `out` (int32[n]
        torch tensor on this graph's device, or a host array)."""
        ptr, where, _keep = _ptr_and_where(out, np.int32)
        d = ctypes.c_int32()
        check(lib().mce_preprocess(self._h, ORIENT[orientation], None, ptr, where, ctypes.byref(d)))
        return out

    def core_into(self, core, peel):
        """Preprocess with the degeneracy orientation (cached) and copy its core
        numbers and peel order into `core` / `peel` (int32[n], both torch tensors
        on this graph's device or both host arrays)."""
        cptr, where, _k1 = _ptr_and_where(core, np.int32)
        pptr, where2, _k2 = _ptr_and_where(peel, np.int32)
        if where != where2:
            raise ValueError("core and peel must both be on the host or both on the device")
        d = ctypes.c_int32()
        check(lib().mce_preprocess(self._h, ORIENT["degeneracy"], cptr, pptr, where, ctypes.byref(d)))
        return core, peel

    def set_core(self, core, peel):
        """mce_set_core: take core numbers and a degeneracy (peel) order computed
        elsewhere (another rank's core_into) instead of peeling here."""
        cptr, where, _k1 = _ptr_and_where(core, np.int32)
        pptr, where2, _k2 = _ptr_and_where(peel, np.int32)
        if where != where2:
            raise ValueError("core and peel must both be on the host or both on the device")
        check(lib().mce_set_core(self._h, cptr, pptr, where))

    def set_order(self, order, orientation: str = "degeneracy"):
        """mce_set_order: orient the edges along `order` (vertex of rank i)."""
        ptr, where, _keep = _ptr_and_where(order, np.int32)
        check(lib().mce_set_order(self._h, ORIENT[orientation], ptr, where))

    def heuristic(self, kind: str = "multi_degree", h: int = 0):
        """(omega_bar, clique in order added, run size per seed vertex (0 = not a seed))."""
        w = ctypes.c_int32()
        ln = ctypes.c_int32()
        clique = np.zeros(self.n + 1, np.int32)
        runs = np.zeros(max(self.n, 1), np.int32)
        check(lib().mce_heuristic(self._h, HEURISTIC[kind], int(h), ctypes.byref(w),
                                  clique.ctypes.data_as(ctypes.c_void_p), ctypes.byref(ln),
                                  runs.ctypes.data_as(ctypes.c_void_p)))
        return int(w.value), clique[: ln.value].tolist(), runs[: self.n]

    def _result(self, handle, cliques: str = "host") -> Result:
        L = lib()
        try:
            om = ctypes.c_int32()
            cnt = ctypes.c_int64()
            st = ctypes.c_int64()
            tr = ctypes.c_int32()
            check(L.mce_result_info(handle, ctypes.byref(om), ctypes.byref(cnt), ctypes.byref(st), ctypes.byref(tr)))
            if cliques == "device":  # the canonical rows stay in HBM: a torch tensor on the graph's device
                if torch is None:
                    raise RuntimeError("cliques='device' needs torch")
                cl = torch.empty((st.value, max(om.value, 0)), dtype=torch.int32,
                                 device=torch.device("cuda", self.device))
                check(L.mce_result_cliques(handle, ctypes.c_void_p(cl.data_ptr()) if cl.numel() else None,
                                           _lib.WHERE_DEVICE))
            else:
                cl = np.empty((st.value, max(om.value, 0)), np.int32)
                check(L.mce_result_cliques(handle, cl.ctypes.data_as(ctypes.c_void_p) if cl.size else None,
                                           _lib.WHERE_HOST))
            nl = ctypes.c_int32()
            ent = (ctypes.c_int64 * 512)()
            check(L.mce_result_levels(handle, ent, 512, ctypes.byref(nl)))
            tm = (ctypes.c_double * 21)()
            check(L.mce_result_timing(handle, tm, 21))
            timing = dict(preprocess_ms=tm[0], heuristic_ms=tm[1], expand_ms=tm[2], count_kernel_ms=tm[3],
                          count_launches=int(tm[4]), count_kernel_bytes=tm[5], kernels=int(tm[6]),
                          root_kernel_ms=tm[7], root_launches=int(tm[8]), root_kernel_bytes=tm[9],
                          host_total_ms=tm[10], host_preprocess_ms=tm[11], host_heuristic_ms=tm[12],
                          syncs=int(tm[13]), host_setup_ms=tm[14], host_enum_ms=tm[15], host_readout_ms=tm[16],
                          root_setup_ms=tm[17], build_kernel_ms=tm[18], build_launches=int(tm[19]),
                          build_kernel_bytes=tm[20])
            return Result(om.value, cnt.value, cl, bool(tr.value), [int(ent[i]) for i in range(min(nl.value, 512))],
                          timing)
        finally:
            L.mce_result_free(handle)

    def enumerate(self, cliques: str = "host", **opts) -> Result:
        """All maximum cliques (mce_enumerate).  cliques='host': numpy rows;
        'device': a torch.int32 tensor in the graph's device memory (no copy to
        the host)."""
        o, keep = make_options(**opts)
        h = ctypes.c_void_p()
        st = lib().mce_enumerate(self._h, ctypes.byref(o), ctypes.byref(h))
        if keep is not None:
            keep.reraise()
        check(st)
        return self._result(h, cliques)

    def find_one(self, window: int = 0, **opts) -> Result:
        o, keep = make_options(**opts)
        h = ctypes.c_void_p()
        st = lib().mce_find_one(self._h, int(window), ctypes.byref(o), ctypes.byref(h))
        if keep is not None:
            keep.reraise()
        check(st)
        return self._result(h)


def empty_cache(device: int = 0) -> None:
    """Return the library's cached device memory of `device` to the driver (mce_empty_cache)."""
    check(lib().mce_empty_cache(int(device)))


def version() -> str:
    return lib().mce_version().decode()
