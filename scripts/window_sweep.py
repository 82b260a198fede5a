#!/usr/bin/env python
"""configs[3]: windowed single-maximum-clique search on dense G(800, 0.5) under
a fixed frontier budget, window-size sweep (PAPER.md IV-E, V-C).

    python scripts/window_sweep.py [--budget-mib 1024] [--reps 3] > profiles/r01_window_sweep_dense800.json

One JSON object: per window size (roots per window; 0 = all roots at once)
the median device-event time of find_one over `reps` runs (graph resident,
preprocessing cache cleared every run, L2 flushed), the omega found, the
widest frontier level and the number of levels.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--budget-mib", type=int, default=1024)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--windows", default="1,4,16,64,256,1024,0")
    args = ap.parse_args()
    import torch

    import paper_conf_ipps_geilpo23_b200 as mce
    from synth import graphs as G

    g = G.make_config("dense800").to("cuda")
    gg = mce.Graph(g.rowptr, g.col)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    budget = args.budget_mib << 20
    out = {"workload": "dense800", "config": "G(800, 0.5) seed 1, find_one", "budget_bytes": budget,
           "edges": g.num_edges, "sweep": []}
    for w in [int(x) for x in args.windows.split(",")]:
        times, res = [], None
        for i in range(args.reps + 1):
            gg.clear_cache()
            flush.zero_()
            torch.cuda.synchronize()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            res = gg.find_one(window=w, budget_bytes=budget)
            e.record()
            torch.cuda.synchronize()
            if i:
                times.append(s.elapsed_time(e))
        out["sweep"].append({"window": w, "ms": statistics.median(times), "omega": res.omega,
                             "max_level_entries": max(res.levels) if res.levels else 0,
                             "levels": len(res.levels)})
    print(json.dumps(out))


if __name__ == "__main__":
    main()
