import os, sys
sys.path.insert(0, '.')
os.environ.update(MCE_SMEM_MIN_W="4", MCE_SMEM_MIN_N="1", MCE_SMEM_PER_ROOT="0")
import paper_conf_ipps_geilpo23_b200 as m
from synth import graphs as G
g = G.rmat(15, 16, 0.57, 0.19, 0.19, seed=5).to("cuda")
cases = [dict(), dict(fused_levels=False), dict(clique_shortcut=False),
         dict(budget_bytes=8 << 20, heuristic="none", fused_levels=False), dict(budget_bytes=64 << 20, heuristic="none", fused_levels=False), dict(budget_bytes=8 << 20, heuristic="none"),
         dict(budget_bytes=24 << 20, heuristic="single_degree")]
for kw in cases:
    gg = m.Graph(g.rowptr, g.col)
    try:
        r = gg.enumerate(**kw)
        print("ok", kw, r.omega, r.count, flush=True)
    except Exception as e:
        print("FAIL", kw, e, flush=True)
        pass
    finally:
        gg.close()
