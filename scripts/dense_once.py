"""One windowed find-one on dense800 (for ncu captures of the expansion kernels)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_geilpo23_b200 as m  # noqa: E402
from synth import graphs as G  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "dense800"
g = G.make_config(cfg, device="cuda") if cfg.startswith("rmat") else G.make_config(cfg).to("cuda")
gg = m.Graph(g.rowptr, g.col)
r = gg.find_one(window=64) if cfg == "dense800" else gg.enumerate(max_cliques=1 << 16)
print(cfg, r.omega, r.count, r.timing["expand_ms"])
