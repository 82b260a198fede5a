"""k-core peel trace of one preprocessing (MCE_KCORE_TRACE): per scan, level k, alive vertices, appended, time."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["MCE_KCORE_TRACE"] = "1"
import paper_conf_ipps_geilpo23_b200 as m  # noqa: E402
from synth import graphs as G  # noqa: E402

cfg = sys.argv[1]
g = G.make_config(cfg, device="cuda") if cfg.startswith("rmat") else G.make_config(cfg).to("cuda")
for ov in (0, 1):
    gg = m.Graph(g.rowptr, g.col)
    r = gg.enumerate(max_cliques=1 << 16, overlap=bool(ov))
    print(cfg, "overlap", ov, r.omega, r.count, r.timing["preprocess_ms"], flush=True)
    gg.close()
