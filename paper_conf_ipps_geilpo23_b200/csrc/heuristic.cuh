#pragma once
#include <vector>

#include "graph.cuh"

namespace mce {
struct HeuristicResult {
    int32_t omega_bar = 0;           // best run size (0 when no runs)
    std::vector<int32_t> clique;     // that run's clique, original ids, in order added
    std::vector<int32_t> run_size;   // per vertex: size of the run it seeded, 0 if not a seed
    double ms = 0.0;
    int64_t kernels = 0;
};
// kind: MCE_HEUR_*; h <= 0 means |V|; runs sharded cyclically when shard_count > 1
// concurrent: run on g->hstream / g->hpool / g->hhost (overlapped with
// preprocessing by the engine; degree kinds only); with_core: the core numbers
// are on the device (stream-ordered before the heuristic) and prune seeds and
// candidates (core + 1 < best)
HeuristicResult run_heuristic(mce_graph *g, int kind, int64_t h, int32_t shard_rank, int32_t shard_count,
                              bool want_runs, bool concurrent = false, bool with_core = false);
}  // namespace mce
