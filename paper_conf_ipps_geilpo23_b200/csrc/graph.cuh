// Device-resident graph handle and the preprocessing entry points.
#pragma once

#include <vector>

#include "common.cuh"

struct mce_graph {
    int device = 0;
    cudaStream_t stream = nullptr;
    int64_t n = 0;
    int64_t nnz = 0;  // 2|E|
    int64_t max_deg = 0;
    mce::DevBuf<int64_t> rowptr;  // [n+1] undirected CSR
    mce::DevBuf<int32_t> col;     // [nnz], rows sorted ascending

    // ---- preprocessing (PAPER.md II-B-2, IV-C), computed lazily ----
    int orientation = -1;          // MCE_ORIENT_* the arrays below were built for
    bool have_core = false;
    mce::DevBuf<int32_t> core;     // [n] core numbers
    mce::DevBuf<int32_t> peel;     // [n] k-core peel order (vertex removed i-th)
    int32_t degeneracy = 0;
    mce::DevBuf<int32_t> order;    // [n] rank -> vertex (orientation order)
    mce::DevBuf<int32_t> rank;     // [n] vertex -> rank
    mce::DevBuf<int32_t> vid;      // [n] CSR id -> vertex (ids of orp/ocol: (core, degree) order, or the rank)
    mce::DevBuf<int32_t> pid;      // [n] vertex -> CSR id
    mce::DevBuf<int64_t> orp;      // [n+1] oriented CSR (edges to higher rank), indexed by CSR id
    mce::DevBuf<int32_t> ocol;     // [nnz/2] out-neighbour CSR ids, rows ascending
    mce::DevBuf<int4> ocol4;       // [n] the same rows padded to 16-byte slots (-1 fill), only when max_out <= 4
    bool have_ocol4 = false;       // ocol4 matches the current orientation
    int32_t max_out = 0;           // largest out-degree
    double t_pre_ms = 0.0;         // device time of the last preprocessing (see preprocess_ms)
    cudaEvent_t pre_ev[2] = {nullptr, nullptr};
    bool pre_pending = false;
    bool pre_overlapped = false;   // set by the engine while the heuristic runs concurrently
    bool order_given = false;      // g->order was set by mce_set_order: orient() keeps it
    bool pre_started = false;      // pre_ev[0] already recorded (the engine ran kcore before preprocess)
    int64_t kernels = 0;           // kernels launched by the last preprocessing

    // ---- reusable memory (no cudaMalloc/cudaFree on the steady-state path) ----
    mce::Pool pool;                // per-phase scratch (reset at the start of every phase)
    std::vector<mce::DevBuf<uint8_t>> wsegs;  // frontier arena segments of mce_enumerate / mce_find_one
    mce::PinnedBuf host;           // pinned staging for small device->host reads (per device, shared)
    // the heuristic overlapped with preprocessing (engine.cu) runs on its own
    // thread, stream, scratch pool and pinned slot
    mce::Pool hpool;
    mce::PinnedBuf hhost{1};
    cudaStream_t hstream = nullptr;
    cudaStream_t pstream = nullptr;  // greatest-priority stream of the overlapped preprocessing
    ~mce_graph() {
        if (hstream) cudaStreamDestroy(hstream);
        if (pstream) cudaStreamDestroy(pstream);
        if (pre_ev[0]) cudaEventDestroy(pre_ev[0]);
        if (pre_ev[1]) cudaEventDestroy(pre_ev[1]);
    }
    mce::DevBuf<uint8_t> misc;     // engine: leaf counter + level chain (persistent)
    mce::DevBuf<int32_t> stage;    // engine: staged leaf cliques of one launch (grow-only)
    mce::DevBuf<int32_t> cstage;   // engine: staged clique completions of one launch (grow-only)
    mce::DevBuf<int64_t> pdesc;    // engine: pair-completion descriptors of one launch (grow-only)
    mce::DevBuf<int32_t> store;    // engine: stored maximum cliques of the run (grow-only)
    mce::DevBuf<uint16_t> wide;    // engine: colouring-order scratch of the wide count pass (grow-only)
};

namespace mce {
// k-core numbers and peel order (cooperative persistent kernel)
void kcore(mce_graph *g);
// rank/order by the requested orientation + oriented CSR with sorted rows
void orient(mce_graph *g, int orientation);
// both (the k-core only for the degeneracy orientations), cached on the handle
void preprocess(mce_graph *g, int orientation);
bool preprocessed(const mce_graph *g, int orientation);
// device time of the last preprocessing (waits for it if still pending)
double preprocess_ms(mce_graph *g);
// orientation from a given order (mce_set_order)
void orient_from(mce_graph *g, int orientation, const int32_t *order, bool on_device);
// core numbers + peel order from another handle (mce_set_core): no peel here
void set_core(mce_graph *g, const int32_t *core, const int32_t *peel, bool on_device);
}  // namespace mce
