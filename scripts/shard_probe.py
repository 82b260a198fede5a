"""Shard / bound-sync probe of one configuration on one GPU (debugging aid):
each shard run alone, with a bound_sync that reports the other shard's best."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from synth import graphs as G
import paper_conf_ipps_geilpo23_b200 as mce
cfg = sys.argv[1]
g = G.make_config(cfg, device="cuda") if cfg.startswith("rmat") else G.make_config(cfg).to("cuda")
gg = mce.Graph(g.rowptr, g.col)
r = gg.enumerate(max_cliques=1 << 16)
om = r.omega
print("full", r.omega, r.count, flush=True)
for k in range(2):
    calls = []
    def sync(best, active, calls=calls):
        calls.append((best, active))
        return max(best, om), (1 if len(calls) < 5 else 0)
    gg.clear_cache()
    r = gg.enumerate(max_cliques=1 << 16, shard_rank=k, shard_count=2, bound_sync=sync)
    print("shard", k, "/2 with the global bound", om, "->", r.omega, r.count, "syncs", len(calls), calls[:3], flush=True)
