"""First-timed-step probe (ba1m): step times around the events bench.py places
between warm-up and the timed region.  mode: flush_timed | flush_all | thread | nvml"""
import sys, threading, time, torch
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
    h0 = time.perf_counter()
    r = graph.enumerate(heuristic="multi_degree", orientation="degeneracy", cliques="device")
    h1 = time.perf_counter()
    b.record(s); torch.cuda.synchronize()
    t = r.timing
    return round(a.elapsed_time(b), 3), round((h1 - h0) * 1e3, 3), round(t["preprocess_ms"], 3), round(t["heuristic_ms"], 3)
mode = sys.argv[1]
stop = threading.Event()
for i in range(14):
    if i == 5 and mode == "thread":
        threading.Thread(target=lambda: stop.wait(100), daemon=True).start()
    if i == 5 and mode == "nvml":
        c = bench.ClockSampler(0).prepare(); c.__enter__()
    if i == 5 and mode == "sleep":
        time.sleep(0.05)
    fl = (mode == "flush_all") or (mode == "flush_timed" and i >= 3) or mode in ("thread", "nvml", "sleep")
    print(mode, i, fl, step(fl))
stop.set()
