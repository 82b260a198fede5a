#!/usr/bin/env python
"""Write tests/golden/<config>.json = (omega, multiplicity) from the CPU oracle ONLY.

    python scripts/make_golden_rmat.py rmat22      # ~15 min on one core
    python scripts/make_golden_rmat.py rmat20      # same recipe at scale 20 (~8 min)
    python scripts/make_golden_rmat.py rmat26s20   # configs[4]'s recipe (50 planted 20-cliques) at scale 20

The R-MAT workloads have too many maximum cliques to store (rmat22: 3 * 2^26
cliques of 223 vertices), so the colouring oracle runs in count-only mode
(oracle.count_max_cliques) with the tight-node rule (mce_oracle.c expand(),
a consequence of the |C|+|P| bound of PAPER.md II-B-3) and a lower bound from
the oracle's own greedy heuristic (oracle.greedy, Algorithm 1, 4096 highest-
degree seeds; a lower bound never changes the answer -- pinned by
tests/test_oracle.py::test_lower_bound_does_not_change_answer).  Nothing here
touches the CUDA path.
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from synth import graphs as G  # noqa: E402


def graph(name):
    if name in ("rmat22", "rmat26"):
        return G.make_config(name), f"synth.graphs.make_config('{name}')"
    if name.startswith("rmat26s"):  # the rmat26 recipe (50 planted 20-cliques) at a scale the oracle finishes
        scale = int(name[7:])
        return (G.make_config("rmat26", scale_override=scale),
                f"synth.graphs.make_config('rmat26', scale_override={scale})")
    scale = int(name[4:])
    return G.rmat(scale, 16, 0.57, 0.19, 0.19, seed=1), f"synth.graphs.rmat({scale}, 16, 0.57, 0.19, 0.19, seed=1)"


def main():
    name = sys.argv[1]
    t0 = time.time()
    g, recipe = graph(name)
    rp, col = g.numpy()
    t1 = time.time()
    lb, _, _ = oracle.greedy(rp, col, np.diff(rp), 4096)
    om, cnt = oracle.count_max_cliques(rp, col, lb=int(lb), bound="color", tight=True)
    t2 = time.time()
    out = {
        "_comment": ["Written by scripts/make_golden_rmat.py from oracle.count_max_cliques (colouring bound, "
                     "tight-node rule, greedy lower bound); never from the CUDA path.",
                     f"Graph: {recipe}."],
        "n": g.n, "edges": g.num_edges, "omega": om, "multiplicity": cnt, "oracle_lower_bound": int(lb),
        "oracle_seconds": round(t2 - t1, 1), "generate_seconds": round(t1 - t0, 1),
    }
    path = os.path.join(ROOT, "tests", "golden", f"{name}.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(path, out)


if __name__ == "__main__":
    main()
