// Engine entry point and the result object behind the C ABI.
#pragma once
#include <vector>

#include "graph.cuh"
#include "mce.h"

struct mce_result {
    int32_t omega = 0;
    int64_t count = 0;     // multiplicity (exact)
    int64_t stored = 0;    // rows available
    int32_t truncated = 0;
    std::vector<int32_t> rows;  // stored * omega original vertex ids (host; find-one / wide rows)
    mce::DevBuf<int32_t> drows; // the same on the device when the read-out ran there (canon.cu)
    int device = 0;
    bool canonical = false;     // rows sorted (each clique ascending, list lexicographic)
    std::vector<int64_t> level_entries;
    double t_pre_ms = 0, t_heur_ms = 0, t_enum_ms = 0, t_expand_ms = 0, t_count_ms = 0, count_bytes = 0;
    int64_t count_launches = 0, kernels = 0;
    double t_root_ms = 0, root_bytes = 0;  // fused root-level kernel
    double t_setup_ms = 0;                 // root colour filter + root / re-root matrix builds
    double t_build_ms = 0, build_bytes = 0;  // root matrix builds (build_adj_block) and their algorithmic bytes
    int64_t build_launches = 0;
    int64_t root_launches = 0;
    double h_total_ms = 0, h_pre_ms = 0, h_heur_ms = 0;  // host wall time of the call / its phases
    double h_setup_ms = 0, h_enum_ms = 0, h_readout_ms = 0;
    int64_t syncs = 0;                                    // host<->device round trips
    int32_t overlapped = 0;                               // heuristic ran concurrently with preprocessing
};

namespace mce {
mce_result *run_engine(mce_graph *g, const mce_options &o, bool find_one);
}
