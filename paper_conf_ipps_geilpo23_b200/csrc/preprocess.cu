// Preprocessing on the device (north star: "k-core/degeneracy ordering and
// edge orientation, done on device").
//
//  * kcore(): core numbers (PAPER.md II-B-2, line 61) by parallel peeling in
//    ONE cooperative persistent launch: at level k every alive vertex with
//    degree <= k is queued (core = k); processing a queued vertex decrements
//    its alive neighbours and queues those that fall to k.  The queue order is
//    a degeneracy order: when v is queued its remaining degree (<= k) counts
//    every neighbour queued after it, so orienting edges along the queue gives
//    out-degree <= core(v) <= degeneracy.
//  * orient(): ranks (degeneracy = queue order, or degree order = PAPER.md
//    IV-C line 131 "keep the edge where the source vertex has lower degree"),
//    and the oriented CSR over ranks with every row sorted ascending, so that
//    "the candidates after v" are exactly v's out-neighbours (IV-C line 133).
#include <cooperative_groups.h>

#include <algorithm>
#include <vector>

#include "graph.cuh"

namespace cg = cooperative_groups;

namespace mce {

namespace {

constexpr int kPeelThreads = 512;

// ctrl layout: [0..2] queue append counters (rotating per sub-round),
//              [3..5] alive-list append counters (rotating per sub-round)
__global__ void __launch_bounds__(kPeelThreads)
    kcore_peel(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col, int32_t *deg,
               int32_t *core, int32_t *queue, int32_t *alive_a, int32_t *alive_b, uint8_t *dead,
               unsigned long long *ctrl) {
    cg::grid_group grid = cg::this_grid();
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
    const int64_t warp = tid >> 5;
    const int64_t nwarps = nthreads >> 5;
    const int lane = threadIdx.x & 31;

    int64_t s = 0;          // sub-round
    int64_t head = 0;       // region to process: [head, region_end)
    int64_t region_end = 0;
    int64_t n_alive = n;
    int32_t *cur = alive_a, *nxt = alive_b;
    int32_t k = 0;
    bool scan = true;
    while (true) {
        unsigned long long *qcnt = ctrl + (s % 3);
        unsigned long long *acnt = ctrl + 3 + (s % 3);
        if (tid == 0) {  // zero the counters of sub-round s+1 (last read before this sub-round began)
            ctrl[(s + 1) % 3] = 0;
            ctrl[3 + (s + 1) % 3] = 0;
        }
        if (scan) {
            for (int64_t i = tid; i < n_alive; i += nthreads) {
                int32_t v = cur[i];
                if (dead[v]) continue;
                if (deg[v] <= k) {
                    unsigned long long p = region_end + atomicAdd(qcnt, 1ull);
                    queue[p] = v;
                    core[v] = k;
                    dead[v] = 1;
                } else {
                    unsigned long long p = atomicAdd(acnt, 1ull);
                    nxt[p] = v;
                }
            }
        } else {
            for (int64_t i = head + warp; i < region_end; i += nwarps) {
                int32_t v = queue[i];
                for (int64_t e = rowptr[v] + lane; e < rowptr[v + 1]; e += 32) {
                    int32_t u = col[e];
                    if (!dead[u]) {
                        int32_t old = atomicSub(deg + u, 1);
                        if (old == k + 1) {
                            unsigned long long p = region_end + atomicAdd(qcnt, 1ull);
                            queue[p] = u;
                            core[u] = k;
                            dead[u] = 1;
                        }
                    }
                }
            }
        }
        grid.sync();
        const int64_t c = (int64_t)(*(volatile unsigned long long *)qcnt);
        if (scan) {
            n_alive = (int64_t)(*(volatile unsigned long long *)acnt);
            int32_t *t = cur;
            cur = nxt;
            nxt = t;
        }
        head = region_end;
        region_end += c;
        if (region_end >= n) break;  // every vertex has its core number
        if (c == 0) {
            ++k;
            scan = true;
        } else {
            scan = false;
        }
        ++s;
    }
}

__global__ void degrees_kernel(int64_t n, const int64_t *__restrict__ rowptr, int32_t *deg, int32_t *iota) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        deg[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
        iota[v] = (int32_t)v;
    }
}

__global__ void invert_kernel(int64_t n, const int32_t *__restrict__ order, int32_t *rank) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        rank[order[i]] = (int32_t)i;
}

// degree order: counting sort by degree (ties in arbitrary order)
__global__ void degree_hist(int64_t n, const int64_t *__restrict__ rowptr, int32_t *bins) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(bins + (rowptr[v + 1] - rowptr[v]), 1);
}
__global__ void degree_scatter(int64_t n, const int64_t *__restrict__ rowptr, unsigned long long *cursor,
                               int32_t *order) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long p = atomicAdd(cursor + (rowptr[v + 1] - rowptr[v]), 1ull);
        order[p] = (int32_t)v;
    }
}

// out-degree of every rank: warp per vertex, ballot over neighbour chunks
__global__ void out_degree_kernel(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                  const int32_t *__restrict__ rank, int32_t *odeg) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t v = warp; v < n; v += nwarps) {
        const int32_t r = rank[v];
        int32_t cnt = 0;
        for (int64_t e0 = rowptr[v]; e0 < rowptr[v + 1]; e0 += 32) {
            int64_t e = e0 + lane;
            bool up = e < rowptr[v + 1] && rank[col[e]] > r;
            cnt += __popc(__ballot_sync(0xffffffffu, up));
        }
        if (lane == 0) odeg[r] = cnt;
    }
}

// fill the oriented rows (in CSR order of the source; sorted afterwards)
__global__ void orient_fill_kernel(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                   const int32_t *__restrict__ rank, const int64_t *__restrict__ orp,
                                   int32_t *ocol) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t v = warp; v < n; v += nwarps) {
        const int32_t r = rank[v];
        int64_t out = orp[r];
        for (int64_t e0 = rowptr[v]; e0 < rowptr[v + 1]; e0 += 32) {
            int64_t e = e0 + lane;
            int32_t ru = e < rowptr[v + 1] ? rank[col[e]] : -1;
            bool up = ru > r;
            unsigned m = __ballot_sync(0xffffffffu, up);
            if (up) ocol[out + __popc(m & lanemask_lt())] = ru;
            out += __popc(m);
        }
    }
}

// ---- row sorts (rows of the oriented CSR) ----
__device__ __forceinline__ int32_t warp_bitonic_sort(int32_t x) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int size = 2; size <= 32; size <<= 1) {
#pragma unroll
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            int32_t y = __shfl_xor_sync(0xffffffffu, x, stride);
            bool up = ((lane & size) == 0);
            bool lower = ((lane & stride) == 0);
            int32_t lo = min(x, y), hi = max(x, y);
            x = (lower == up) ? lo : hi;
        }
    }
    return x;
}

__global__ void sort_rows_warp(int64_t n, const int64_t *__restrict__ orp, int32_t *ocol) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t r = warp; r < n; r += nwarps) {
        int64_t b = orp[r], len = orp[r + 1] - b;
        if (len <= 1 || len > 32) continue;
        int32_t x = lane < len ? ocol[b + lane] : INT32_MAX;
        x = warp_bitonic_sort(x);
        if (lane < len) ocol[b + lane] = x;
    }
}

// one block per long row, bitonic network over the next power of two.
// buf: shared memory when it fits, else a global scratch of `cap` ints.
__global__ void sort_rows_block(const int64_t *__restrict__ orp, int32_t *ocol, const int32_t *__restrict__ rows,
                                int32_t nrows, int32_t *gscratch, int32_t smem_cap) {
    extern __shared__ int32_t smem[];
    for (int32_t ri = blockIdx.x; ri < nrows; ri += gridDim.x) {
        int32_t r = rows[ri];
        int64_t b = orp[r], len = orp[r + 1] - b;
        int32_t p2 = 1;
        while (p2 < len) p2 <<= 1;
        int32_t *buf = p2 <= smem_cap ? smem : gscratch;
        for (int32_t i = threadIdx.x; i < p2; i += blockDim.x) buf[i] = i < len ? ocol[b + i] : INT32_MAX;
        __syncthreads();
        for (int32_t size = 2; size <= p2; size <<= 1) {
            for (int32_t stride = size >> 1; stride > 0; stride >>= 1) {
                for (int32_t i = threadIdx.x; i < p2; i += blockDim.x) {
                    int32_t j = i ^ stride;
                    if (j > i) {
                        bool up = (i & size) == 0;
                        int32_t a = buf[i], c = buf[j];
                        if ((a > c) == up) {
                            buf[i] = c;
                            buf[j] = a;
                        }
                    }
                }
                __syncthreads();
            }
        }
        for (int32_t i = threadIdx.x; i < len; i += blockDim.x) ocol[b + i] = buf[i];
        __syncthreads();
    }
}

__global__ void long_rows_kernel(int64_t n, const int64_t *__restrict__ orp, int32_t *rows, int32_t *count,
                                 int32_t *max_out) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        int32_t len = (int32_t)(orp[r + 1] - orp[r]);
        atomicMax(max_out, len);
        if (len > 32) rows[atomicAdd(count, 1)] = (int32_t)r;
    }
}

}  // namespace

int num_sms() {
    static int sms = 0;
    if (!sms) {
        int dev;
        MCE_CUDA(cudaGetDevice(&dev));
        MCE_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    }
    return sms;
}

int grid_for(int64_t work_items, int threads_per_block, int max_blocks_per_sm) {
    int64_t want = ceil_div(work_items > 0 ? work_items : 1, threads_per_block);
    int64_t cap = (int64_t)num_sms() * max_blocks_per_sm;
    return (int)std::max<int64_t>(1, std::min(want, cap));
}

void kcore(mce_graph *g) {
    if (g->have_core) return;
    const int64_t n = g->n;
    cudaStream_t s = g->stream;
    g->core.alloc(std::max<int64_t>(n, 1));
    g->peel.alloc(std::max<int64_t>(n, 1));
    if (n == 0) {
        g->have_core = true;
        g->degeneracy = 0;
        return;
    }
    DevBuf<int32_t> deg(n), alive_a(n), alive_b(n);
    DevBuf<uint8_t> dead(n);
    DevBuf<unsigned long long> ctrl(8);
    MCE_CUDA(cudaMemsetAsync(dead.get(), 0, n, s));
    MCE_CUDA(cudaMemsetAsync(ctrl.get(), 0, ctrl.bytes(), s));
    degrees_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), deg.get(), alive_a.get());
    MCE_LAUNCH_CHECK();
    int blocks_per_sm = 0;
    MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, kcore_peel, kPeelThreads, 0));
    blocks_per_sm = std::max(1, std::min(blocks_per_sm, 4));
    int grid = num_sms() * blocks_per_sm;
    int64_t n_arg = n;
    const int64_t *rp = g->rowptr.get();
    const int32_t *cl = g->col.get();
    int32_t *dg = deg.get(), *co = g->core.get(), *qu = g->peel.get(), *aa = alive_a.get(), *ab = alive_b.get();
    uint8_t *dd = dead.get();
    unsigned long long *ct = ctrl.get();
    void *args[] = {&n_arg, &rp, &cl, &dg, &co, &qu, &aa, &ab, &dd, &ct};
    MCE_CUDA(cudaLaunchCooperativeKernel((void *)kcore_peel, grid, kPeelThreads, args, 0, s));
    g->kernels += 2;
    // degeneracy = max core (the last queued vertex has it)
    int32_t last_v = 0;
    MCE_CUDA(cudaMemcpyAsync(&last_v, g->peel.get() + n - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    MCE_CUDA(cudaStreamSynchronize(s));
    MCE_CUDA(cudaMemcpy(&g->degeneracy, g->core.get() + last_v, sizeof(int32_t), cudaMemcpyDeviceToHost));
    g->have_core = true;
}

void orient(mce_graph *g, int orientation) {
    if (g->orientation == orientation) return;
    const int64_t n = g->n;
    cudaStream_t s = g->stream;
    g->order.alloc(std::max<int64_t>(n, 1));
    g->rank.alloc(std::max<int64_t>(n, 1));
    g->orp.alloc(n + 1);
    g->ocol.alloc(std::max<int64_t>(g->nnz / 2, 1));
    if (n == 0) {
        MCE_CUDA(cudaMemsetAsync(g->orp.get(), 0, sizeof(int64_t), s));
        g->orientation = orientation;
        g->max_out = 0;
        return;
    }
    if (orientation == 0) {  // degeneracy: the peel queue
        MCE_CUDA(cudaMemcpyAsync(g->order.get(), g->peel.get(), sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
    } else {  // degree order
        int64_t nb = g->max_deg + 1;
        DevBuf<int32_t> bins(nb);
        DevBuf<int64_t> cursor(nb + 1), tmp(scan_tmp_items(nb));
        MCE_CUDA(cudaMemsetAsync(bins.get(), 0, bins.bytes(), s));
        degree_hist<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), bins.get());
        MCE_LAUNCH_CHECK();
        exclusive_scan_i32(bins.get(), cursor.get(), nb, tmp.get(), s);
        degree_scatter<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(),
                                                         (unsigned long long *)cursor.get(), g->order.get());
        MCE_LAUNCH_CHECK();
        MCE_CUDA(cudaStreamSynchronize(s));
        g->kernels += 5;
    }
    invert_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->order.get(), g->rank.get());
    MCE_LAUNCH_CHECK();
    DevBuf<int32_t> odeg(n);
    out_degree_kernel<<<grid_for(n * 32, 256), 256, 0, s>>>(n, g->rowptr.get(), g->col.get(), g->rank.get(),
                                                            odeg.get());
    MCE_LAUNCH_CHECK();
    {
        DevBuf<int64_t> tmp(scan_tmp_items(n));
        exclusive_scan_i32(odeg.get(), g->orp.get(), n, tmp.get(), s);
    }
    orient_fill_kernel<<<grid_for(n * 32, 256), 256, 0, s>>>(n, g->rowptr.get(), g->col.get(), g->rank.get(),
                                                             g->orp.get(), g->ocol.get());
    MCE_LAUNCH_CHECK();
    sort_rows_warp<<<grid_for(n * 32, 256), 256, 0, s>>>(n, g->orp.get(), g->ocol.get());
    MCE_LAUNCH_CHECK();
    DevBuf<int32_t> rows(n), meta(2);
    MCE_CUDA(cudaMemsetAsync(meta.get(), 0, meta.bytes(), s));
    long_rows_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->orp.get(), rows.get(), meta.get(), meta.get() + 1);
    MCE_LAUNCH_CHECK();
    int32_t hmeta[2];
    MCE_CUDA(cudaMemcpyAsync(hmeta, meta.get(), sizeof(hmeta), cudaMemcpyDeviceToHost, s));
    MCE_CUDA(cudaStreamSynchronize(s));
    g->kernels += 8;
    g->max_out = hmeta[1];
    if (hmeta[0] > 0) {
        const int32_t smem_cap = 8192;  // ints (32 KB)
        int32_t p2 = 1;
        while (p2 < g->max_out) p2 <<= 1;
        if (p2 <= smem_cap) {
            sort_rows_block<<<grid_for(hmeta[0], 1, 16), 256, smem_cap * sizeof(int32_t), s>>>(
                g->orp.get(), g->ocol.get(), rows.get(), hmeta[0], nullptr, smem_cap);
            MCE_LAUNCH_CHECK();
        } else {  // some row exceeds shared memory: one block, global scratch
            DevBuf<int32_t> scratch(p2);
            sort_rows_block<<<1, 1024, smem_cap * sizeof(int32_t), s>>>(g->orp.get(), g->ocol.get(), rows.get(),
                                                                        hmeta[0], scratch.get(), smem_cap);
            MCE_LAUNCH_CHECK();
            MCE_CUDA(cudaStreamSynchronize(s));
        }
        g->kernels += 1;
    }
    MCE_CUDA(cudaStreamSynchronize(s));
    g->orientation = orientation;
}

void preprocess(mce_graph *g, int orientation) {
    if (g->have_core && g->orientation == orientation) return;
    cudaEvent_t e0, e1;
    MCE_CUDA(cudaEventCreate(&e0));
    MCE_CUDA(cudaEventCreate(&e1));
    MCE_CUDA(cudaEventRecord(e0, g->stream));
    g->kernels = 0;
    kcore(g);
    orient(g, orientation);
    MCE_CUDA(cudaEventRecord(e1, g->stream));
    MCE_CUDA(cudaEventSynchronize(e1));
    float ms = 0;
    MCE_CUDA(cudaEventElapsedTime(&ms, e0, e1));
    g->t_pre_ms = ms;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
}

}  // namespace mce
