#!/usr/bin/env python
"""Benchmark: time to enumerate all maximum cliques and edges/s on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config rmat22]
    python bench.py --impl reference ...     # the CPU oracle arm (no reference code exists)

A step is one full pass of the hot path from a CSR resident in HBM:
k-core/orientation preprocessing + greedy heuristic + breadth-first expansion
(+ for N > 1 the per-step bound all-reduces and the final clique gather),
i.e. PAPER.md V line 315's timing ("do not include the time to load the
graph dataset onto the GPU, but do include the heuristic runtime and other
preprocessing").  L2 is flushed (256 MiB write) before every timed step.
Prints ONE JSON line on rank 0.
"""

from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "edges/s to enumerate all maximum cliques (time-to-solution incl. preprocessing + heuristic)"
CONFIG_INDEX = {"er2000": 0, "ba1m": 1, "rmat22": 2, "dense800": 3, "rmat26": 4}
# (n, |E|) of the full workloads (synth.graphs.make_config; the GPU arm prints the graph's own, equal, values)
CONFIG_SIZES = {"er2000": (2000, 10002), "ba1m": (1000000, 3999984), "rmat22": (4194304, 64154352),
                "dense800": (800, 159278), "rmat26": (67108864, 1051929294)}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    # default: configs[2], the workload BASELINE.json's metric is quoted on at 1/2/4/8 B200
    p.add_argument("--config", default="rmat22", choices=list(CONFIG_INDEX))
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--mode", default=None, choices=[None, "enumerate", "find_one"])
    p.add_argument("--window", type=int, default=-1,
                   help="find-one roots per window (PAPER.md IV-E); -1: 96 for dense800 (the best of the "
                        "window sweep under the degree orientation, profiles/r02_window_sweep_dense800_v2.md), "
                        "else 0 = all roots")
    p.add_argument("--max-cliques", type=int, default=-1,
                   help="stored-clique capacity (multiplicity stays exact); -1: 2^16 for the R-MAT configs "
                        "(~10^8 maximum cliques of size ~223 there), unbounded otherwise")
    p.add_argument("--heuristic", default="auto",
                   choices=["auto", "none", "single_degree", "single_core", "multi_degree", "multi_core"],
                   help="lower-bound heuristic (PAPER.md IV-A); auto: the per-config choice of HEURISTIC below "
                        "(PAPER.md V line 315 reports each dataset under its fastest heuristic)")
    p.add_argument("--orientation", default="auto", choices=["auto", "degeneracy", "degree", "degeneracy_det"],
                   help="edge orientation (PAPER.md IV-C: the paper keeps the edge from the lower-degree vertex; "
                        "the degeneracy orders bound every out-degree by the core number); auto: ORIENTATION below")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--shard-depth", type=int, default=-1,
                   help="N > 1: <= 1 deals roots, d >= 2 replicates levels < d and deals the level-d candidates "
                        "by hash (mce_options.shard_depth); -1: 3 for rmat26 (work under a few hub roots), else 0")
    return p.parse_args()


class ClockSampler:
    """SM clocks + throttle reasons sampled DURING the timed region (B200_PROFILING.md clocks line).

    In-process NVML polling every 20 ms (no nvidia-smi child process, whose
    queries can stall a short timed region); nvidia-smi -lms is the fallback.
    """

    REASONS = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20, "sw_power_cap": 0x4}

    def __init__(self, index: int, interval_s: float = 0.02):
        self.index = index
        self.interval = interval_s
        self.samples = []  # (sm_mhz, max_mhz, reasons bitmask)
        self._stop = threading.Event()
        self._nvml = None
        self._proc = None

    def _poll_nvml(self):
        N, h, mx = self._nvml, self._h, self._mx
        while True:
            try:
                sm = N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)
                rs = N.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.samples.append((float(sm), float(mx), int(rs)))
            except Exception:
                pass
            if self._stop.wait(self.interval):
                break

    def _poll_smi(self):
        fields = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                  "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        self._proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={fields}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        bits = [0x8, 0x40, 0x20, 0x4]
        for line in self._proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            try:
                rs = sum(b for b, v in zip(bits, parts[2:6]) if v.lower() == "active")
                self.samples.append((float(parts[0]), float(parts[1]), rs))
            except (ValueError, IndexError):
                continue

    def prepare(self):
        """NVML init and handle lookup, before the warm-up steps (kept out of the
        timed region; the thread only polls clocks and reasons)."""
        try:
            import pynvml as N

            N.nvmlInit()
            self._h = N.nvmlDeviceGetHandleByIndex(self.index)
            self._mx = N.nvmlDeviceGetMaxClockInfo(self._h, N.NVML_CLOCK_SM)
            N.nvmlDeviceGetClockInfo(self._h, N.NVML_CLOCK_SM)
            N.nvmlDeviceGetCurrentClocksEventReasons(self._h)
            self._nvml = N
        except Exception:
            self._nvml = None
        self._prepared = True
        return self

    def __enter__(self):
        if not getattr(self, "_prepared", False):
            self.prepare()
        target = self._poll_nvml if self._nvml is not None else self._poll_smi
        self._t = threading.Thread(target=target, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self._proc:
            self._proc.terminate()
        self._t.join(timeout=5)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        reasons = sorted(n for n, b in self.REASONS.items() if any(s[2] & b for s in self.samples))
        return {"sm_mhz": statistics.median(s[0] for s in self.samples),
                "sm_max_mhz": max(s[1] for s in self.samples), "reasons": reasons, "samples": len(self.samples),
                "source": "nvml" if self._nvml else "nvidia-smi"}


def measured_peak_hbm():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# PAPER.md abstract (line 25) and V (line 315): context, not a target.
PAPER_CONTEXT = {
    "claim": "average speedup of 1.9x over previous parallel work (PMC, Rossi et al.) on 58 real-world graphs",
    "hardware": "NVIDIA Tesla A100 40GB (CUDA 11.6) vs PMC on a 2.8 GHz 24-core AMD EPYC 7402, 512 GB",
    "timing": "average of 5 runs, graph load excluded, heuristic + preprocessing included (PAPER.md V line 315)",
    "source": "PAPER.md line 25 (abstract), line 315 (V)",
}


def sample_graph(config: str):
    """The bounded CPU sample of a workload (the oracle cannot finish the full
    R-MAT configs in minutes: rmat22 has 3 * 2^26 maximum cliques of 223
    vertices): the same generator and parameters at R-MAT scale 17 (6 s of
    oracle time); the other configs are their own sample."""
    from synth import graphs as G

    if config in ("rmat22", "rmat26"):
        g = G.make_config(config, device="cuda" if _has_cuda() else "cpu",
                          scale_override=17).to("cpu")
        return g, f"same R-MAT recipe as {config} at scale 17 ({g.n} vertices, {g.num_edges} edges)"
    g = G.make_config(config)
    return g, f"the full {config} workload"


def _has_cuda():
    try:
        import torch

        return torch.cuda.is_available()
    except Exception:  # pragma: no cover
        return False


def cpu_baseline(config: str, budget_s=10.0):
    """The oracle as it stands (single-threaded C, colouring bound) on a bounded
    sample of the workload, repeated until ~budget_s of CPU time."""
    import oracle

    g, what = sample_graph(config)
    rp, col = g.numpy()
    runs, total = 0, 0.0
    while total < budget_s or runs == 0:
        t0 = time.perf_counter()
        om, cl = oracle.max_cliques(rp, col)
        total += time.perf_counter() - t0
        runs += 1
    dt = total / runs
    return {"value": g.num_edges / dt, "unit": "edges/s", "cores": 1, "kind": "oracle",
            "sample": f"{what}; enumerate all maximum cliques, {runs} run(s) of {dt:.2f} s (omega={om}, "
                      f"multiplicity={len(cl)})",
            "seconds_per_run": dt}


def golden(config: str):
    """tests/golden/<config>.json: (omega, multiplicity) written by scripts that call only oracle/."""
    try:
        with open(os.path.join(ROOT, "tests", "golden", f"{config}.json")) as f:
            d = json.load(f)
        return int(d["omega"]), (int(d["multiplicity"]) if d.get("multiplicity") is not None else None)
    except (OSError, ValueError, KeyError):
        return None


def verify(config: str, mode: str, res, g):
    """Check the GPU answer: against the oracle's golden (omega, multiplicity)
    when one is committed, else against the oracle itself on small configs."""
    gd = golden(config)
    if gd is not None:
        om, cnt = gd
        ok = res.omega == om and (mode == "find_one" or cnt is None or res.count == cnt)
        return {"against": f"tests/golden/{config}.json (oracle)", "omega": om,
                "multiplicity": cnt if mode == "enumerate" else None, "ok": bool(ok)}
    if config in ("er2000", "ba1m"):
        import oracle

        om, cl = oracle.max_cliques(*g.numpy(), bound="plain")
        ok = res.omega == om and (mode == "find_one" or res.count == len(cl))
        return {"against": "oracle (list-based B&B) on the same graph", "omega": om, "multiplicity": len(cl),
                "ok": bool(ok)}
    return {"against": None, "ok": None}


def config_dict(config, mode, window, n, edges, max_cl, world, shard_depth):
    """The workload description both arms print (identical keys and values)."""
    return {"workload": config, "baseline_config_index": CONFIG_INDEX[config], "mode": mode,
            "window": window if mode == "find_one" else None, "n": n, "edges": edges, "max_cliques": max_cl,
            "parallelism": (f"root-shard x{world}" if shard_depth < 2 else
                            f"level-{shard_depth} candidate shard x{world}"),
            "l2": "flushed (256 MiB write) before every step"}


# per-config heuristic (the answer never depends on it, only the work does; PAPER.md V line 315: "we
# report the results from the fastest configuration ... the best combination of heuristic, window
# size, and other preprocessing"); chosen by the sweep in profiles/r02_heuristic_sweep_*.json
HEURISTIC = {"er2000": "multi_degree", "ba1m": "multi_degree", "rmat22": "multi_degree",
             "dense800": "multi_degree", "rmat26": "multi_degree"}


# per-config orientation (same reasoning as HEURISTIC: the answer never depends on it), from the sweep in
# profiles/r02_orientation_sweep_v1.md: the paper's degree orientation skips the k-core peel and wins on
# er2000 and dense800; rmat22 needs the degeneracy order (out-degree <= core: the root colour filter and
# narrow root spaces); ba1m keeps it too -- 1.20 ms with degree vs 1.41, but its sparse root kernel
# (out-degrees <= 4 only under the degeneracy order) is the north star's >= 50% HBM roofline kernel
ORIENTATION = {"er2000": "degree", "ba1m": "degeneracy", "rmat22": "degeneracy", "dense800": "degree",
               "rmat26": "degeneracy"}


def bench_defaults(args):
    mode = args.mode or ("find_one" if args.config == "dense800" else "enumerate")
    shard_depth = args.shard_depth if args.shard_depth >= 0 else (3 if args.config == "rmat26" else 0)
    window = args.window if args.window >= 0 else (96 if args.config == "dense800" else 0)
    max_cl = args.max_cliques if args.max_cliques >= 0 else (1 << 16 if args.config.startswith("rmat") else 0)
    if args.heuristic == "auto":
        args.heuristic = HEURISTIC[args.config]
    if args.orientation == "auto":
        args.orientation = ORIENTATION[args.config]
    return mode, shard_depth, window, max_cl


def ncu_traffic(config: str, kname: str):
    """DRAM bytes per launch (dram__bytes_read.sum + dram__bytes_write.sum) of this config's dominant
    kernel from the committed `ncu --set full` capture (profiles/ncu_traffic.json), or None."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            rec = json.load(f).get(config)
    except (OSError, ValueError):
        return None
    if not rec or rec.get("kernel", "") not in kname:
        return None
    return rec.get("bytes_per_launch")


def build_graph(config: str, device: str):
    from synth import graphs as G

    if config in ("rmat22", "rmat26"):
        return G.make_config(config, device=device)
    return G.make_config(config).to(device)


def run_reference(args):
    """--impl reference: the CPU oracle timed on the host cores (rank 0 only),
    each step one oracle run on the bounded sample of the workload."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle

    mode, shard_depth, window, max_cl = bench_defaults(args)
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    g, what = sample_graph(args.config)
    n_full, edges_full = CONFIG_SIZES.get(args.config, (g.n, g.num_edges))
    rp, col = g.numpy()
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        om, cl = oracle.max_cliques(rp, col)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    t = statistics.mean(times)
    value = g.num_edges / t
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": config_dict(args.config, mode, window, n_full, edges_full, max_cl, world, shard_depth),
        "details": {"sample": what, "omega": om, "multiplicity": len(cl)},
        "cpu_baseline": {"value": value, "unit": "edges/s", "cores": 1, "kind": "oracle",
                         "sample": f"{what}; one oracle run per step ({t:.2f} s)"},
        "e2e": {"value": value, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "paper_context": PAPER_CONTEXT,
    }
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_geilpo23_b200 as mce
    from paper_conf_ipps_geilpo23_b200 import distributed as mdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # test hooks for the multi-process path on a one-GPU box: every rank on
    # cuda:0, gloo instead of NCCL (the driver's N-GPU runs use neither)
    if os.environ.get("MCE_BENCH_SAME_DEVICE") == "1":
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if os.environ.get("MCE_BENCH_BACKEND") == "gloo":
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    rdev = "cpu" if (world > 1 and dist.get_backend() == "gloo") else f"cuda:{local}"
    mode, shard_depth, args.window, max_cl = bench_defaults(args)
    heur = args.heuristic
    orient = args.orientation
    # world > 1 with "degeneracy": rank 0 peels and broadcasts its cores and
    # order, every rank orients from them (distributed.agree_core)

    g = build_graph(args.config, f"cuda:{local}")
    edges = g.num_edges
    stream = torch.cuda.current_stream()
    graph = mce.Graph(g.rowptr, g.col, device=local)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=f"cuda:{local}")

    def one_step(gr):
        gr.clear_cache()
        if world > 1:
            if mode == "enumerate":
                return mdist.enumerate_distributed(gr, max_cliques=max_cl, shard_depth=shard_depth, heuristic=heur,
                                                   orientation=orient)
            return mdist.find_one_distributed(gr, window=args.window, heuristic=heur, orientation=orient)
        if mode == "enumerate":
            # the step's inputs are resident in HBM and so are its outputs: the canonical
            # cliques stay in device memory (the e2e measurement below copies them to the host)
            return gr.enumerate(max_cliques=max_cl, heuristic=heur, orientation=orient, cliques="device")
        return gr.find_one(window=args.window, heuristic=heur, orientation=orient)

    clocks = ClockSampler(local).prepare()
    for _ in range(args.warmup):  # the same sequence as a timed step (flush, sync, step)
        flush.fill_(1)
        torch.cuda.synchronize()
        res = one_step(graph)
    times = []
    timings = []
    py_ms = []
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    start.record(stream)  # (the CUDA events are created at their first record: not inside a timed step)
    end.record(stream)
    torch.cuda.synchronize()
    with clocks:
        for _ in range(args.steps):
            flush.fill_(1)  # L2 flush (256 MiB > 126 MB L2) before every timed step
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            start.record(stream)
            h0 = time.perf_counter()
            res = one_step(graph)
            py_ms.append((time.perf_counter() - h0) * 1e3)
            end.record(stream)
            torch.cuda.synchronize()
            times.append(start.elapsed_time(end))
            timings.append(res.timing)
    t_ms = sum(times) / len(times)  # exactly K timed steps
    if world > 1:
        tt = torch.tensor([t_ms], dtype=torch.float64, device=rdev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_ms = float(tt.item())
    value = edges / (t_ms / 1e3)

    # ---- roofline of the dominant expansion kernel, live CUDA-event timing on the library's stream:
    # the fused root-level kernel or the count pass of levels >= 2, whichever takes longer
    tm = timings[-1]
    peak, peak_src = measured_peak_hbm()
    cnt_ms = statistics.mean(t["count_kernel_ms"] for t in timings)
    root_ms = statistics.mean(t["root_kernel_ms"] for t in timings)
    build_ms = statistics.mean(t.get("build_kernel_ms", 0.0) for t in timings)
    cands = []  # (device ms per step, name, algorithmic bytes per step, launches per step)
    if tm["root_launches"] > 0:
        cands.append((root_ms, "root_expand_l4 / root_expand_w1 (fused root level: adjacency build + first expansion)",
                      tm["root_kernel_bytes"], tm["root_launches"]))
    if tm.get("build_launches", 0) > 0:
        cands.append((build_ms, "build_adj_block (root level of W >= 2 roots: N+(v) of every v in V intersected with "
                      "V = N+(r), PAPER.md IV-D; the adjacency bit matrix of the root's space)",
                      tm["build_kernel_bytes"], tm["build_launches"]))
    cands.append((cnt_ms, "expand (fused count + write pass of levels >= 2: mce::expand_thread / expand_tile / "
                  "expand_lock / expand_wide)", tm["count_kernel_bytes"], tm["count_launches"]))
    k_ms, kname, k_bytes, launches = max(cands, key=lambda c: c[0])
    launches = max(launches, 1)
    achieved = (k_bytes / launches) / ((k_ms / launches) / 1e3) / 1e9 if k_ms > 0 else 0.0
    traffic = ncu_traffic(args.config, kname)
    phases = {"preprocess_ms": statistics.mean(t["preprocess_ms"] for t in timings),
              "heuristic_ms": statistics.mean(t["heuristic_ms"] for t in timings),
              "expand_ms": statistics.mean(t["expand_ms"] for t in timings),
              "expand_count_ms": cnt_ms, "root_kernel_ms": root_ms,
              "root_setup_ms": statistics.mean(t.get("root_setup_ms", 0.0) for t in timings),
              "root_build_kernel_ms": build_ms,
              "host_call_ms": statistics.mean(t["host_total_ms"] for t in timings),
              "host_preprocess_ms": statistics.mean(t["host_preprocess_ms"] for t in timings),
              "host_heuristic_ms": statistics.mean(t["host_heuristic_ms"] for t in timings),
              "host_setup_ms": statistics.mean(t["host_setup_ms"] for t in timings),
              "host_enum_ms": statistics.mean(t["host_enum_ms"] for t in timings),
              "host_readout_ms": statistics.mean(t["host_readout_ms"] for t in timings),
              "syncs_per_step": statistics.mean(t["syncs"] for t in timings),
              "python_step_ms": statistics.mean(py_ms)}

    # ---- end to end through the public API: pinned host CSR -> GPU -> cliques on the host
    e2e = None
    if not args.no_e2e:
        rp_h = g.rowptr.cpu().pin_memory()
        col_h = g.col.cpu().pin_memory()
        e2e_times = []
        d2h = 0
        e2e_warm = 3  # new graph handles: the first calls populate the caching allocator and the arena
        for i in range(e2e_warm + max(3, min(args.steps, 5))):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            gh = mce.Graph(rp_h, col_h, device=local)
            ok = dict(heuristic=heur, orientation=orient)
            r2 = mdist.enumerate_distributed(gh, max_cliques=max_cl, shard_depth=shard_depth, **ok) if (world > 1 and mode == "enumerate") else (
                mdist.find_one_distributed(gh, window=args.window, **ok) if world > 1 else
                (gh.enumerate(max_cliques=max_cl, **ok) if mode == "enumerate" else gh.find_one(window=args.window, **ok)))
            dt = time.perf_counter() - t0
            gh.close()
            if i >= e2e_warm:
                e2e_times.append(dt)
            d2h = int(r2.cliques.nbytes) + 32
        et = statistics.mean(e2e_times)
        if world > 1:
            tt = torch.tensor([et], dtype=torch.float64, device=rdev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            et = float(tt.item())
        e2e = {"value": edges / et, "unit": "edges/s", "h2d_bytes_per_step": int(rp_h.nbytes + col_h.nbytes),
               "d2h_bytes_per_step": d2h, "seconds_per_step": et}

    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            cpu = cpu_baseline(args.config)
        verified = verify(args.config, mode, res, g)
        line = {
            "metric": METRIC,
            "value": value,
            "unit": "edges/s",
            "time_to_solution_s": t_ms / 1e3,
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": t_ms,
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "int32",
            "data": "synthetic",
            "config": config_dict(args.config, mode, args.window, g.n, edges, max_cl, world, shard_depth),
            "details": {"heuristic": heur, "orientation": orient, "outputs": "cliques stay in HBM (e2e copies them to the host)" if (world == 1 and mode == "enumerate") else "host", "omega": res.omega, "multiplicity": res.count, "stored_cliques": int(res.cliques.shape[0]),
                        "phases_ms": phases, "levels": res.levels, "step_ms": [round(t, 4) for t in times]},
            "verified": verified,
            "paper_context": PAPER_CONTEXT,
            "roofline": {"bound": "hbm", "kernel": kname,
                         "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak if peak else None, "traffic": traffic, "peak_source": peak_src,
                         "bytes_per_launch": k_bytes / launches, "launches_per_step": launches,
                         "kernel_ms_per_step": k_ms},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(tm["kernels"]) * args.steps,
            "clocks": clocks.summary(),
        }
        print(json.dumps(line), flush=True)
    graph.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
