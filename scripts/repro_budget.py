"""Repeat the small-budget enumerations of test_smem_expand_widths[RMAT15-8-tile] and report any failure
(the k-core peel order differs run to run, so a budget failure can be intermittent)."""
import os
import sys
import traceback

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.update(MCE_SMEM_KIND="tile", MCE_SMEM_MIN_W="8", MCE_SMEM_MIN_N="1", MCE_SMEM_PER_ROOT="0")
import paper_conf_ipps_geilpo23_b200 as m  # noqa: E402
from synth import graphs as G  # noqa: E402

g = G.rmat(15, 16, 0.57, 0.19, 0.19, seed=5).to("cuda")
cases = [dict(), dict(fused_levels=False), dict(clique_shortcut=False),
         dict(budget_bytes=8 << 20, heuristic="none", fused_levels=False),
         dict(budget_bytes=24 << 20, heuristic="single_degree")]
fails = 0
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 20):
    for kw in cases:
        gg = m.Graph(g.rowptr, g.col)
        try:
            r = gg.enumerate(**kw)
        except Exception as e:  # noqa: BLE001
            fails += 1
            print("FAIL", it, kw, e)
            if fails <= 2:
                gg.close()
                gg = m.Graph(g.rowptr, g.col)
                try:
                    gg.enumerate(verbose=2, **kw)
                except Exception as e2:  # noqa: BLE001
                    print("verbose rerun:", e2)
        finally:
            gg.close()
print("fails", fails)
