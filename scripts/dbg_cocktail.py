import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.test_gpu_parity import cocktail_join, run_enum
import oracle
j, t = int(sys.argv[1]), int(sys.argv[2])
g = cocktail_join(j, t, seed=j * 1000 + t)
om, cl = oracle.max_cliques(*g.numpy())
print("oracle", om, len(cl), flush=True)
for sc in (True, False):
    for fused in (True, False):
        for legacy in (False,):
            r = run_enum(g, clique_shortcut=sc, fused_levels=fused, verbose=1)
            print("shortcut", sc, "fused", fused, "->", r.omega, r.count, flush=True)
