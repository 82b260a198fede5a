"""Probe configs[4] (R-MAT scale 26 + 50 planted 20-cliques) on one GPU: build time, graph shape, enumeration."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from synth import graphs as G
import paper_conf_ipps_geilpo23_b200 as mce

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 26
t = time.time()
g = G.make_config("rmat26", device="cuda", scale_override=scale)
torch.cuda.synchronize()
print(f"built scale {scale}: n={g.n} edges={g.col.numel() // 2} in {time.time() - t:.1f} s", flush=True)
print("deg", G.degree_stats(g), flush=True)
t = time.time()
gg = mce.Graph(g.rowptr, g.col)
del g
torch.cuda.empty_cache()
print(f"loaded in {time.time() - t:.1f} s", flush=True)
for rep in range(2):
    t = time.time()
    r = gg.enumerate(max_cliques=1 << 16, verbose=1 if rep == 0 else 0)
    print(f"enumerate: omega={r.omega} count={r.count} stored={r.cliques.shape} in {time.time() - t:.2f} s "
          f"timing={ {k: v for k, v in r.timing.items() if 'ms' in k} }", flush=True)
