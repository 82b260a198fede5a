"""A/B of one config under environment settings, one process, same graph: python scripts/ab_env.py <config> VAR=a,VAR=b ..."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_geilpo23_b200 as m  # noqa: E402
from synth import graphs as G  # noqa: E402

cfg = sys.argv[1]
g = G.make_config(cfg, device="cuda") if cfg.startswith("rmat") else G.make_config(cfg).to("cuda")
reps = int(os.environ.get("AB_REPS", "1"))
for spec in sys.argv[2:]:
    env = dict(kv.split("=") for kv in spec.split(",") if kv)
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    for rep in range(reps):
        gg = m.Graph(g.rowptr, g.col)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = gg.find_one(window=64) if cfg == "dense800" else gg.enumerate(max_cliques=1 << 16)
        dt = time.perf_counter() - t0
        tm = r.timing
        print(f"{spec or 'default'} rep{rep}: {dt * 1e3:.1f} ms omega {r.omega} count {r.count} setup {tm['root_setup_ms']:.1f} pre {tm['preprocess_ms']:.1f} "
              f"heur {tm['heuristic_ms']:.1f} enum(host) {tm['host_enum_ms']:.1f} expand {tm['expand_ms']:.1f}", flush=True)
        gg.close()
    for k, v in old.items():
        if v is None:
            os.environ.pop(k)
        else:
            os.environ[k] = v
