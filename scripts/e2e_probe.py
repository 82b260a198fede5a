"""Break the bench's e2e step (pinned host CSR -> Graph -> enumerate -> cliques on the host -> close) into phases."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_geilpo23_b200 as mce
from synth import graphs as G

cfg = sys.argv[1] if len(sys.argv) > 1 else "ba1m"
g = G.make_config(cfg)
rp = g.rowptr.pin_memory()
col = g.col.pin_memory()
for i in range(6):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    gh = mce.Graph(rp, col)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    r = gh.enumerate(max_cliques=(1 << 16) if cfg.startswith("rmat") else 0)
    t2 = time.perf_counter()
    gh.close()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    print(f"{cfg} load {1e3*(t1-t0):.2f} ms  enumerate {1e3*(t2-t1):.2f} ms (lib host {r.timing['host_total_ms']:.2f})  close {1e3*(t3-t2):.2f} ms", flush=True)
