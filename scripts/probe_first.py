import sys, time, torch
sys.path.insert(0, '.')
import bench
import paper_conf_ipps_geilpo23_b200 as mce
g = bench.build_graph("ba1m", "cuda:0")
graph = mce.Graph(g.rowptr, g.col, device=0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:0")
s = torch.cuda.current_stream()
def step(fl):
    if fl: flush.fill_(1)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s); graph.clear_cache()
    r = graph.enumerate(heuristic="multi_degree", orientation="degeneracy", cliques="device")
    b.record(s); torch.cuda.synchronize()
    t = r.timing
    return round(a.elapsed_time(b), 3), round(t["preprocess_ms"], 3), round(t["heuristic_ms"], 3), round(t.get("host_preprocess_ms", 0), 3), round(t.get("host_heuristic_ms", 0), 3)
mode = sys.argv[1]
for i in range(14):
    fl = (mode == "flush_all") or (mode == "flush_timed" and i >= 3)
    print(i, fl, step(fl))
