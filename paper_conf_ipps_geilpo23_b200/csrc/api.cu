// C ABI of libmce_b200 (declared in include/mce.h).  Argument checking,
// status codes, graph upload and result read-out; all compute is in the
// kernels of preprocess.cu, heuristic.cu, expand.cu.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <string>
#include <thread>
#include <vector>

#include "engine.cuh"
#include "heuristic.cuh"

namespace mce {
namespace {
thread_local std::string g_last_error;
}
void fail(int status, const std::string &msg) { throw Error(status, msg); }

namespace {
// validation: rows sorted strictly ascending, ids in range, no loops, symmetric
__global__ void validate_kernel(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                int32_t *bad) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = rowptr[v], e = rowptr[v + 1];
        if (e < b) {
            atomicOr(bad, 1);
            continue;
        }
        for (int64_t i = b; i < e; ++i) {
            const int32_t u = col[i];
            if (u < 0 || u >= n) {
                atomicOr(bad, 2);
                break;
            }
            if (u == v) atomicOr(bad, 4);
            if (i > b && col[i - 1] >= u) atomicOr(bad, 8);
            if (!contains_sorted(col, rowptr[u], rowptr[u + 1], (int32_t)v)) atomicOr(bad, 16);
        }
    }
}
// largest degree: per-thread max, warp max, one atomic per warp
__global__ void max_deg_kernel(int64_t n, const int64_t *__restrict__ rowptr, unsigned long long *out) {
    unsigned long long m = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        m = max(m, (unsigned long long)(rowptr[v + 1] - rowptr[v]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}



template <typename F>
mce_status run_guarded(F &&f) {
    try {
        f();
        return MCE_OK;
    } catch (const Error &e) {
        g_last_error = e.what();
        return (mce_status)e.status;
    } catch (const std::bad_alloc &) {
        g_last_error = "host allocation failed";
        return MCE_ERR_NOMEM;
    } catch (const std::exception &e) {
        g_last_error = e.what();
        return MCE_ERR_INVALID;
    }
}

void canonicalize(mce_result *r) {
    if (r->canonical) return;  // already ordered on the device (canon.cu)
    if (r->omega <= 0 || r->stored <= 1) {
        if (r->omega > 0)
            for (int64_t i = 0; i < r->stored; ++i)
                std::sort(r->rows.begin() + i * r->omega, r->rows.begin() + (i + 1) * r->omega);
        r->canonical = true;
        return;
    }
    const int32_t k = r->omega;
    for (int64_t i = 0; i < r->stored; ++i) std::sort(r->rows.begin() + i * k, r->rows.begin() + (i + 1) * k);
    std::vector<int64_t> idx(r->stored);
    std::iota(idx.begin(), idx.end(), 0);
    const int32_t *d = r->rows.data();
    std::sort(idx.begin(), idx.end(), [d, k](int64_t a, int64_t b) {
        return std::lexicographical_compare(d + a * k, d + (a + 1) * k, d + b * k, d + (b + 1) * k);
    });
    std::vector<int32_t> out((size_t)r->stored * k);
    for (int64_t i = 0; i < r->stored; ++i) std::memcpy(out.data() + i * k, d + idx[i] * k, sizeof(int32_t) * k);
    r->rows.swap(out);
    r->canonical = true;
}
}  // namespace
}  // namespace mce

using namespace mce;

extern "C" {

const char *mce_last_error(void) { return g_last_error.c_str(); }
const char *mce_version(void) { return "mce_b200 0.1 (sm_100a)"; }

void mce_default_options(mce_options *o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->orientation = MCE_ORIENT_DEGENERACY;
    o->heuristic = MCE_HEUR_MULTI_DEGREE;
    o->heuristic_runs = 0;
    o->bound = MCE_BOUND_COLOR;
    o->lower_bound = 0;
    o->window = 0;
    o->budget_bytes = 0;
    o->max_cliques = 0;
    o->shard_rank = 0;
    o->shard_count = 1;
    o->bound_sync = nullptr;
    o->bound_sync_user = nullptr;
    o->verbose = 0;
    o->legacy_roots = 0;
    o->no_fused_levels = 0;
    o->no_clique_shortcut = 0;
    o->no_fused_expand = 0;
    o->no_overlap = 0;
    o->no_smem_expand = 0;
    o->no_reroot = 0;
    o->shard_depth = 0;
}

mce_status mce_load_csr(int32_t device, int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int32_t where,
                        int32_t validate, void *stream, mce_graph **out) {
    return run_guarded([&] {
        if (!out) fail(MCE_ERR_INVALID, "out is NULL");
        *out = nullptr;
        if (n < 0 || n >= (1ll << 31)) fail(MCE_ERR_INVALID, "n out of range");
        if (!row_ptr) fail(MCE_ERR_INVALID, "row_ptr is NULL");
        if (where != MCE_WHERE_HOST && where != MCE_WHERE_DEVICE) fail(MCE_ERR_INVALID, "bad `where`");
        int ndev = 0;
        MCE_CUDA(cudaGetDeviceCount(&ndev));
        if (device < 0 || device >= ndev) fail(MCE_ERR_INVALID, "bad device index");
        MCE_CUDA(cudaSetDevice(device));
        int major = 0;  // (cudaGetDeviceProperties costs milliseconds: one attribute instead)
        MCE_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device));
        if (major < 10) fail(MCE_ERR_CUDA, "libmce_b200 needs an sm_100 (Blackwell) device");
        const bool trace = getenv("MCE_TRACE_LOAD") != nullptr;
        using lclk = std::chrono::steady_clock;
        const auto t0 = lclk::now();
        auto lap = [&](const char *what) {
            if (trace)
                fprintf(stderr, "[mce] load %s %.3f ms\n", what,
                        std::chrono::duration<double, std::milli>(lclk::now() - t0).count());
        };
        auto g = new mce_graph();
        try {
            g->device = device;
            g->stream = (cudaStream_t)stream;
            g->n = n;
            int64_t nnz = 0;
            auto kind = where == MCE_WHERE_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
            if (where == MCE_WHERE_HOST)
                nnz = row_ptr[n];
            else
                MCE_CUDA(cudaMemcpy(&nnz, row_ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost));
            if (nnz < 0 || (nnz & 1)) fail(MCE_ERR_INVALID, "row_ptr[n] must be 2|E| (even, >= 0)");
            if (nnz > 0 && !col_idx) fail(MCE_ERR_INVALID, "col_idx is NULL");
            g->nnz = nnz;
            lap("start");
            g->rowptr.alloc(n + 1);
            g->col.alloc(std::max<int64_t>(nnz, 1));
            lap("alloc");
            MCE_CUDA(cudaMemcpyAsync(g->rowptr.get(), row_ptr, sizeof(int64_t) * (n + 1), kind, g->stream));
            if (nnz)
                MCE_CUDA(cudaMemcpyAsync(g->col.get(), col_idx, sizeof(int32_t) * nnz, kind, g->stream));
            lap("copies issued");
            if (n > 0) {
                g->pool.reset();
                unsigned long long *md = g->pool.take<unsigned long long>(1);
                MCE_CUDA(cudaMemsetAsync(md, 0, sizeof(unsigned long long), g->stream));
                max_deg_kernel<<<grid_for(n, 256), 256, 0, g->stream>>>(n, g->rowptr.get(), md);
                MCE_LAUNCH_CHECK();
                unsigned long long *h = g->host.get<unsigned long long>(1);
                MCE_CUDA(cudaMemcpyAsync(h, md, sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream));
                stream_sync(g->stream);
                lap("copied + max degree");
                g->max_deg = (int64_t)h[0];
                if (validate) {
                    int32_t *bad = g->pool.take<int32_t>(1);
                    MCE_CUDA(cudaMemsetAsync(bad, 0, sizeof(int32_t), g->stream));
                    validate_kernel<<<grid_for(n, 256), 256, 0, g->stream>>>(n, g->rowptr.get(), g->col.get(), bad);
                    MCE_LAUNCH_CHECK();
                    int32_t *hbp = g->host.get<int32_t>(1);
                    MCE_CUDA(cudaMemcpyAsync(hbp, bad, sizeof(int32_t), cudaMemcpyDeviceToHost, g->stream));
                    stream_sync(g->stream);
                    const int32_t hb = hbp[0];
                    if (hb)
                        fail(MCE_ERR_INVALID, "malformed CSR (flags " + std::to_string(hb) +
                                                  ": 1 rowptr, 2 id range, 4 loop, 8 unsorted/dup, 16 asymmetric)");
                }
            }
            stream_sync(g->stream);
        } catch (...) {
            delete g;
            throw;
        }
        *out = g;
    });
}

void mce_graph_free(mce_graph *g) { delete g; }

mce_status mce_graph_clear_cache(mce_graph *g) {
    return run_guarded([&] {
        if (!g) fail(MCE_ERR_INVALID, "graph is NULL");
        g->have_core = false;
        g->orientation = -1;
    });
}

mce_status mce_set_order(mce_graph *g, int32_t orientation, const int32_t *order, int32_t where) {
    return run_guarded([&] {
        if (!g) fail(MCE_ERR_INVALID, "graph is NULL");
        if (orientation != MCE_ORIENT_DEGENERACY && orientation != MCE_ORIENT_DEGREE)
            fail(MCE_ERR_INVALID, "bad orientation");
        if (!order && g->n) fail(MCE_ERR_INVALID, "order is NULL");
        MCE_CUDA(cudaSetDevice(g->device));
        orient_from(g, orientation, order, where == MCE_WHERE_DEVICE);
    });
}

mce_status mce_set_core(mce_graph *g, const int32_t *core, const int32_t *peel, int32_t where) {
    return run_guarded([&] {
        if (!g) fail(MCE_ERR_INVALID, "graph is NULL");
        if ((!core || !peel) && g->n) fail(MCE_ERR_INVALID, "core or peel is NULL");
        MCE_CUDA(cudaSetDevice(g->device));
        set_core(g, core, peel, where == MCE_WHERE_DEVICE);
    });
}

mce_status mce_preprocess(mce_graph *g, int32_t orientation, int32_t *core_out, int32_t *order_out, int32_t where,
                          int32_t *degeneracy_out) {
    return run_guarded([&] {
        if (!g) fail(MCE_ERR_INVALID, "graph is NULL");
        if (orientation < MCE_ORIENT_DEGENERACY || orientation > MCE_ORIENT_DEGENERACY_DET)
            fail(MCE_ERR_INVALID, "bad orientation");
        MCE_CUDA(cudaSetDevice(g->device));
        preprocess(g, orientation);
        if (core_out || degeneracy_out) kcore(g);  // (the degree orientation does not need them)
        auto kind = where == MCE_WHERE_HOST ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
        if (core_out && g->n) MCE_CUDA(cudaMemcpy(core_out, g->core.get(), sizeof(int32_t) * g->n, kind));
        if (order_out && g->n) MCE_CUDA(cudaMemcpy(order_out, g->order.get(), sizeof(int32_t) * g->n, kind));
        if (degeneracy_out) *degeneracy_out = g->degeneracy;
    });
}

mce_status mce_heuristic(mce_graph *g, int32_t kind, int64_t h, int32_t *omega_bar_out, int32_t *clique_out,
                         int32_t *clique_len_out, int32_t *run_size_out) {
    return run_guarded([&] {
        if (!g) fail(MCE_ERR_INVALID, "graph is NULL");
        if (kind < MCE_HEUR_NONE || kind > MCE_HEUR_MULTI_CORE) fail(MCE_ERR_INVALID, "bad heuristic kind");
        MCE_CUDA(cudaSetDevice(g->device));
        HeuristicResult r = run_heuristic(g, kind, h, 0, 1, run_size_out != nullptr);
        if (omega_bar_out) *omega_bar_out = r.omega_bar;
        if (clique_len_out) *clique_len_out = (int32_t)r.clique.size();
        if (clique_out && !r.clique.empty()) std::memcpy(clique_out, r.clique.data(), sizeof(int32_t) * r.clique.size());
        if (run_size_out) {
            if (r.run_size.empty())
                std::memset(run_size_out, 0, sizeof(int32_t) * g->n);
            else
                std::memcpy(run_size_out, r.run_size.data(), sizeof(int32_t) * g->n);
        }
    });
}

static void check_options(const mce_options *o) {
    if (!o) fail(MCE_ERR_INVALID, "options are NULL");
    if (o->orientation < MCE_ORIENT_DEGENERACY || o->orientation > MCE_ORIENT_DEGENERACY_DET)
        fail(MCE_ERR_INVALID, "bad orientation");
    if (o->heuristic < MCE_HEUR_NONE || o->heuristic > MCE_HEUR_MULTI_CORE) fail(MCE_ERR_INVALID, "bad heuristic");
    if (o->bound != MCE_BOUND_SIZE && o->bound != MCE_BOUND_COLOR) fail(MCE_ERR_INVALID, "bad bound");
    if (o->shard_count > 1 && (o->shard_rank < 0 || o->shard_rank >= o->shard_count))
        fail(MCE_ERR_INVALID, "bad shard rank");
}

mce_status mce_enumerate(mce_graph *g, const mce_options *opt, mce_result **out) {
    return run_guarded([&] {
        if (!g || !out) fail(MCE_ERR_INVALID, "NULL argument");
        *out = nullptr;
        mce_options o;
        if (opt)
            o = *opt;
        else
            mce_default_options(&o);
        check_options(&o);
        MCE_CUDA(cudaSetDevice(g->device));
        *out = run_engine(g, o, false);
    });
}

mce_status mce_find_one(mce_graph *g, int64_t window, const mce_options *opt, mce_result **out) {
    return run_guarded([&] {
        if (!g || !out) fail(MCE_ERR_INVALID, "NULL argument");
        *out = nullptr;
        mce_options o;
        if (opt)
            o = *opt;
        else
            mce_default_options(&o);
        if (window > 0) o.window = window;
        check_options(&o);
        MCE_CUDA(cudaSetDevice(g->device));
        *out = run_engine(g, o, true);
    });
}

mce_status mce_result_info(const mce_result *r, int32_t *omega, int64_t *count, int64_t *stored,
                           int32_t *truncated) {
    return run_guarded([&] {
        if (!r) fail(MCE_ERR_INVALID, "result is NULL");
        if (omega) *omega = r->omega;
        if (count) *count = r->count;
        if (stored) *stored = r->stored;
        if (truncated) *truncated = r->truncated;
    });
}

mce_status mce_result_cliques(mce_result *r, int32_t *dst, int32_t where) {
    return run_guarded([&] {
        if (!r) fail(MCE_ERR_INVALID, "result is NULL");
        const size_t bytes = sizeof(int32_t) * (size_t)r->stored * std::max(r->omega, 0);
        if (r->drows.get()) {  // canonical rows on the device
            if (!bytes) return;
            if (!dst) fail(MCE_ERR_INVALID, "dst is NULL");
            MCE_CUDA(cudaSetDevice(r->device));
            if (where != MCE_WHERE_HOST) {
                MCE_CUDA(cudaMemcpy(dst, r->drows.get(), bytes, cudaMemcpyDeviceToDevice));
                return;
            }
            if (bytes < (8u << 20)) {
                MCE_CUDA(cudaMemcpy(dst, r->drows.get(), bytes, cudaMemcpyDeviceToHost));
                return;
            }
            // large: through the cached pinned staging at full link speed, in
            // chunks, the host copies of a chunk spread over threads and
            // overlapped with the next chunk's transfer
            constexpr size_t kChunkBytes = 32u << 20;
            char *stage = static_cast<char *>(mce::host_pinned(2 * kChunkBytes));
            cudaStream_t st;
            MCE_CUDA(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
            cudaEvent_t ev[2];
            MCE_CUDA(cudaEventCreateWithFlags(&ev[0], cudaEventDisableTiming));
            MCE_CUDA(cudaEventCreateWithFlags(&ev[1], cudaEventDisableTiming));
            const char *src = reinterpret_cast<const char *>(r->drows.get());
            char *out = reinterpret_cast<char *>(dst);
            const size_t nchunks = (bytes + kChunkBytes - 1) / kChunkBytes;
            auto issue = [&](size_t c) {
                const size_t off = c * kChunkBytes, len = std::min(kChunkBytes, bytes - off);
                MCE_CUDA(cudaMemcpyAsync(stage + (c & 1) * kChunkBytes, src + off, len, cudaMemcpyDeviceToHost, st));
                MCE_CUDA(cudaEventRecord(ev[c & 1], st));
            };
            issue(0);
            for (size_t c = 0; c < nchunks; ++c) {
                if (c + 1 < nchunks) issue(c + 1);
                MCE_CUDA(cudaEventSynchronize(ev[c & 1]));
                const size_t off = c * kChunkBytes, len = std::min(kChunkBytes, bytes - off);
                const char *from = stage + (c & 1) * kChunkBytes;
                const int nt = 8;
                std::vector<std::thread> th;
                const size_t part = (len + nt - 1) / nt;
                for (int t = 0; t < nt; ++t) {
                    const size_t b = t * part;
                    if (b >= len) break;
                    th.emplace_back([=] { std::memcpy(out + off + b, from + b, std::min(part, len - b)); });
                }
                for (auto &x : th) x.join();

            }
            cudaEventDestroy(ev[0]);
            cudaEventDestroy(ev[1]);
            cudaStreamDestroy(st);
            return;
        }
        canonicalize(r);
        if (!bytes) return;
        if (!dst) fail(MCE_ERR_INVALID, "dst is NULL");
        if (where == MCE_WHERE_HOST)
            std::memcpy(dst, r->rows.data(), bytes);
        else
            MCE_CUDA(cudaMemcpy(dst, r->rows.data(), bytes, cudaMemcpyHostToDevice));
    });
}

mce_status mce_result_levels(const mce_result *r, int64_t *entries, int32_t cap, int32_t *levels_out) {
    return run_guarded([&] {
        if (!r) fail(MCE_ERR_INVALID, "result is NULL");
        int32_t L = (int32_t)r->level_entries.size();
        if (levels_out) *levels_out = L;
        for (int32_t i = 0; i < std::min(cap, L) && entries; ++i) entries[i] = r->level_entries[i];
    });
}

mce_status mce_result_timing(const mce_result *r, double *t, int32_t cap) {
    return run_guarded([&] {
        if (!r || !t) fail(MCE_ERR_INVALID, "NULL argument");
        double v[21] = {r->t_pre_ms,    r->t_heur_ms,     r->t_expand_ms,          r->t_count_ms,
                        (double)r->count_launches, r->count_bytes, (double)r->kernels, r->t_root_ms,
                        (double)r->root_launches,  r->root_bytes,  r->h_total_ms, r->h_pre_ms,
                        r->h_heur_ms,              (double)r->syncs, r->h_setup_ms, r->h_enum_ms,
                        r->h_readout_ms,           r->t_setup_ms,    r->t_build_ms,
                        (double)r->build_launches, r->build_bytes};
        for (int32_t i = 0; i < std::min(cap, 21); ++i) t[i] = v[i];
    });
}

void mce_result_free(mce_result *r) { delete r; }

}  // extern "C"
