#!/usr/bin/env python
"""Write tests/golden/dense800.json from the CPU oracle ONLY (never the CUDA path).

    python scripts/make_golden.py

dense800 = BASELINE.json configs[3]: G(n=800, p=0.5) seed 1 (synth.graphs).
The oracle's full enumeration takes ~30 s single-threaded, too long for the
CPU test suite, so the answer is stored here and the GPU find-one test checks
omega against it (and the clique against the definition).
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from synth import graphs as G  # noqa: E402


def main():
    g = G.make_config("dense800")
    rp, col = g.numpy()
    t0 = time.time()
    om, cl = oracle.max_cliques(rp, col)
    dt = time.time() - t0
    out = {
        "_comment": ["Written by scripts/make_golden.py from oracle.max_cliques (colouring bound).",
                     "Graph: synth.graphs.make_config('dense800') = G(800, 0.5) seed 1 (BASELINE.json configs[3])."],
        "n": g.n, "edges": g.num_edges, "omega": om, "multiplicity": int(len(cl)),
        "cliques": cl.tolist(), "oracle_seconds": round(dt, 2),
    }
    path = os.path.join(ROOT, "tests", "golden", "dense800.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(path, om, len(cl), f"{dt:.1f}s")


if __name__ == "__main__":
    main()
