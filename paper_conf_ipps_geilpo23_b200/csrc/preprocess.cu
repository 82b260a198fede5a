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

// ctrl layout (rotating per sub-round s, index s % 3):
//   [0..2] queue append counters, [3..5] alive-list append counters,
//   [6..8] smallest degree among the vertices a scan kept alive
//
// Level-synchronous peel: a "scan" sub-round queues every alive vertex with
// degree <= k and compacts the rest into the next alive list; a "cascade"
// sub-round processes the vertices queued by the previous sub-round (one warp
// per vertex, lanes over its neighbours) and queues neighbours whose degree
// falls to k.  All appends are warp-aggregated (one atomicAdd per warp and
// ballot ranks), so no counter sees more than one atomic per warp.  When a
// scan queues nothing, k jumps straight to the smallest alive degree it saw.
__device__ __forceinline__ unsigned long long warp_append(unsigned long long *ctr, unsigned mask, int lane) {
    unsigned long long base = 0;
    if (lane == 0 && mask) base = atomicAdd(ctr, (unsigned long long)__popc(mask));
    return __shfl_sync(0xffffffffu, base, 0);
}

// cascade step for one queued vertex v by a tile of G lanes: decrement the
// alive neighbours, queue those that fall to k (one atomicAdd per tile chunk)
template <int G>
__device__ __forceinline__ void peel_neighbours(int32_t v, const int64_t *__restrict__ rowptr,
                                                const int32_t *__restrict__ col, int32_t *deg, int32_t *core,
                                                int32_t *queue, uint8_t *dead, unsigned long long *qcnt,
                                                int64_t region_end, int32_t k) {
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1), gbase = lane & ~(G - 1);
    const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
    const int64_t eb = rowptr[v], ee = rowptr[v + 1];
    for (int64_t e0 = eb; e0 < ee; e0 += G) {
        const int64_t e = e0 + gl;
        bool fell = false;
        int32_t u = -1;
        if (e < ee) {
            u = col[e];
            if (!dead[u]) fell = atomicSub(deg + u, 1) == k + 1;
        }
        const unsigned fm = (__ballot_sync(gmask, fell) & gmask) >> gbase;
        if (fm) {
            unsigned long long b = 0;
            if (gl == 0) b = atomicAdd(qcnt, (unsigned long long)__popc(fm));
            b = __shfl_sync(gmask, b, 0, G);
            if (fell) {
                queue[region_end + b + __popc(fm & ((1u << gl) - 1u))] = u;
                core[u] = k;
                dead[u] = 1;
            }
        }
    }
}

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
    const unsigned lt = lanemask_lt();

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
        unsigned long long *mind = ctrl + 6 + (s % 3);
        if (tid == 0) {  // reset the counters of sub-round s+1 (last read before this sub-round began)
            ctrl[(s + 1) % 3] = 0;
            ctrl[3 + (s + 1) % 3] = 0;
            ctrl[6 + (s + 1) % 3] = ~0ull;
        }
        if (scan) {
            int32_t dmin = INT32_MAX;
            for (int64_t i0 = warp * 32; i0 < n_alive; i0 += nwarps * 32) {
                const int64_t i = i0 + lane;
                int32_t v = -1, d = 0;
                bool live = false;
                if (i < n_alive) {
                    v = cur[i];
                    live = !dead[v];
                    if (live) d = deg[v];
                }
                const bool q = live && d <= k;
                const bool keep = live && d > k;
                const unsigned qm = __ballot_sync(0xffffffffu, q);
                const unsigned km = __ballot_sync(0xffffffffu, keep);
                const unsigned long long qb = warp_append(qcnt, qm, lane);
                const unsigned long long kb = warp_append(acnt, km, lane);
                if (q) {
                    queue[region_end + qb + __popc(qm & lt)] = v;
                    core[v] = k;
                    dead[v] = 1;
                }
                if (keep) {
                    nxt[kb + __popc(km & lt)] = v;
                    dmin = min(dmin, d);
                }
            }
            dmin = __reduce_min_sync(0xffffffffu, dmin);
            if (lane == 0 && dmin != INT32_MAX) atomicMin(mind, (unsigned long long)dmin);
        } else {
            // warp takes four queued vertices: 8-lane tiles when all have degree <= 64
            for (int64_t q0 = head + warp * 4; q0 < region_end; q0 += nwarps * 4) {
                const int64_t qi = q0 + (lane >> 3);
                const int32_t v = qi < region_end ? queue[qi] : -1;
                const int64_t d = v >= 0 ? rowptr[v + 1] - rowptr[v] : 0;
                if (__all_sync(0xffffffffu, d <= 64)) {
                    if (v >= 0) peel_neighbours<8>(v, rowptr, col, deg, core, queue, dead, qcnt, region_end, k);
                } else {
                    for (int t = 0; t < 4; ++t) {
                        const int32_t vt = __shfl_sync(0xffffffffu, v, 8 * t);
                        if (vt < 0) break;
                        peel_neighbours<32>(vt, rowptr, col, deg, core, queue, dead, qcnt, region_end, k);
                    }
                }
                __syncwarp();
            }
        }
        grid.sync();
        const int64_t c = (int64_t)(*(volatile unsigned long long *)qcnt);
        const unsigned long long md = *(volatile unsigned long long *)mind;
        const bool was_scan = scan;
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
            // a scan that queued nothing saw every alive degree: jump to the smallest
            k = was_scan ? (int32_t)md : k + 1;
            scan = true;
        } else {
            scan = false;
        }
        ++s;
    }
}

// degeneracy = core number of the last vertex peeled
__global__ void last_core_kernel(int64_t n, const int32_t *__restrict__ peel, const int32_t *__restrict__ core,
                                 int32_t *out) {
    out[0] = core[peel[n - 1]];
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

// Tile of G lanes (8 or 32) inside a warp: lane index, first lane, member mask.
template <int G>
struct Tile {
    int gl, gbase;
    unsigned mask;
    __device__ Tile() {
        const int lane = threadIdx.x & 31;
        gl = lane & (G - 1);
        gbase = lane & ~(G - 1);
        mask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
    }
    __device__ unsigned ballot(bool p) const { return (__ballot_sync(mask, p) & mask) >> gbase; }
    __device__ unsigned lt() const { return (1u << gl) - 1u; }
};

// out-degree of vertex v's rank (tile of G lanes over v's neighbours)
template <int G>
__device__ void out_degree_one(int64_t v, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                               const int32_t *__restrict__ rank, int32_t *odeg) {
    Tile<G> t;
    const int32_t r = rank[v];
    int32_t cnt = 0;
    const int64_t eb = rowptr[v], ee = rowptr[v + 1];
    for (int64_t e0 = eb; e0 < ee; e0 += G) {
        const int64_t e = e0 + t.gl;
        cnt += __popc(t.ballot(e < ee && rank[col[e]] > r));
    }
    if (t.gl == 0) odeg[r] = cnt;
}

// oriented row of v (in CSR order of the source; sorted afterwards)
template <int G>
__device__ void orient_fill_one(int64_t v, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                const int32_t *__restrict__ rank, const int64_t *__restrict__ orp, int32_t *ocol) {
    Tile<G> t;
    const int32_t r = rank[v];
    int64_t out = orp[r];
    const int64_t eb = rowptr[v], ee = rowptr[v + 1];
    for (int64_t e0 = eb; e0 < ee; e0 += G) {
        const int64_t e = e0 + t.gl;
        const int32_t ru = e < ee ? rank[col[e]] : -1;
        const bool up = ru > r;
        const unsigned m = t.ballot(up);
        if (up) ocol[out + __popc(m & t.lt())] = ru;
        out += __popc(m);
    }
}

// Warp w takes vertices [4w, 4w+4): 8-lane tiles when all four have degree
// <= 64 (sparse graphs: a warp per vertex would leave most lanes idle),
// otherwise one vertex after another on the whole warp.
template <bool FILL>
__global__ void __launch_bounds__(256) orient_kernel(int64_t n, const int64_t *__restrict__ rowptr,
                                                     const int32_t *__restrict__ col, const int32_t *__restrict__ rank,
                                                     int32_t *odeg, const int64_t *__restrict__ orp, int32_t *ocol) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t v0 = warp * 4; v0 < n; v0 += nwarps * 4) {
        const int64_t v = v0 + (lane >> 3);
        const int64_t d = v < n ? rowptr[v + 1] - rowptr[v] : 0;
        if (__all_sync(0xffffffffu, d <= 64)) {
            if (v < n) {
                if (FILL)
                    orient_fill_one<8>(v, rowptr, col, rank, orp, ocol);
                else
                    out_degree_one<8>(v, rowptr, col, rank, odeg);
            }
        } else {
            for (int t = 0; t < 4 && v0 + t < n; ++t) {
                if (FILL)
                    orient_fill_one<32>(v0 + t, rowptr, col, rank, orp, ocol);
                else
                    out_degree_one<32>(v0 + t, rowptr, col, rank, odeg);
            }
        }
        __syncwarp();
    }
}

// ---- row sorts (rows of the oriented CSR) ----
// bitonic sort of G values held one per lane of a G-lane tile (ascending)
template <int G>
__device__ __forceinline__ int32_t tile_bitonic_sort(int32_t x, unsigned mask) {
    const int gl = threadIdx.x & (G - 1);
#pragma unroll
    for (int size = 2; size <= G; size <<= 1) {
#pragma unroll
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            int32_t y = __shfl_xor_sync(mask, x, stride, G);
            bool up = ((gl & size) == 0);
            bool lower = ((gl & stride) == 0);
            int32_t lo = min(x, y), hi = max(x, y);
            x = (lower == up) ? lo : hi;
        }
    }
    return x;
}

// rows of length <= 32: 8-lane tiles for four rows of length <= 8, else a warp per row
__global__ void __launch_bounds__(256) sort_rows_warp(int64_t n, const int64_t *__restrict__ orp, int32_t *ocol) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t r0 = warp * 4; r0 < n; r0 += nwarps * 4) {
        const int64_t r = r0 + (lane >> 3);
        const int64_t b = r < n ? orp[r] : 0, len = r < n ? orp[r + 1] - b : 0;
        if (__all_sync(0xffffffffu, len <= 8)) {
            Tile<8> t;
            int32_t x = t.gl < len ? ocol[b + t.gl] : INT32_MAX;
            x = tile_bitonic_sort<8>(x, t.mask);
            if (t.gl < len && len > 1) ocol[b + t.gl] = x;
        } else {
            for (int q = 0; q < 4; ++q) {
                const int64_t bb = __shfl_sync(0xffffffffu, b, 8 * q);
                const int64_t ll = __shfl_sync(0xffffffffu, len, 8 * q);
                if (ll <= 1 || ll > 32) continue;
                int32_t x = lane < ll ? ocol[bb + lane] : INT32_MAX;
                x = tile_bitonic_sort<32>(x, 0xffffffffu);
                if (lane < ll) ocol[bb + lane] = x;
            }
        }
        __syncwarp();
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

// rows longer than a warp (sorted by one block each) and the largest out-degree
__global__ void long_rows_kernel(int64_t n, const int64_t *__restrict__ orp, int32_t *rows, int32_t *count,
                                 int32_t *max_out) {
    const int lane = threadIdx.x & 31;
    int32_t mx = 0;
    for (int64_t r0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) & ~31ll; r0 < n;
         r0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = r0 + lane;
        const int32_t len = r < n ? (int32_t)(orp[r + 1] - orp[r]) : 0;
        mx = max(mx, len);
        const unsigned m = __ballot_sync(0xffffffffu, len > 32);
        int32_t b = 0;
        if (lane == 0 && m) b = atomicAdd(count, __popc(m));
        b = __shfl_sync(0xffffffffu, b, 0);
        if (len > 32) rows[b + __popc(m & lanemask_lt())] = (int32_t)r;
    }
    mx = __reduce_max_sync(0xffffffffu, mx);
    if (lane == 0 && mx) atomicMax(max_out, mx);
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
    g->core.ensure(std::max<int64_t>(n, 1));
    g->peel.ensure(std::max<int64_t>(n, 1));
    if (n == 0) {
        g->have_core = true;
        g->degeneracy = 0;
        return;
    }
    g->pool.reset();
    int32_t *deg = g->pool.take<int32_t>(n), *alive_a = g->pool.take<int32_t>(n), *alive_b = g->pool.take<int32_t>(n);
    uint8_t *dead = g->pool.take<uint8_t>(n);
    unsigned long long *ctrl = g->pool.take<unsigned long long>(9);
    MCE_CUDA(cudaMemsetAsync(dead, 0, n, s));
    MCE_CUDA(cudaMemsetAsync(ctrl, 0, 6 * sizeof(unsigned long long), s));
    MCE_CUDA(cudaMemsetAsync(ctrl + 6, 0xff, 3 * sizeof(unsigned long long), s));
    degrees_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), deg, alive_a);
    MCE_LAUNCH_CHECK();
    int blocks_per_sm = 0;
    MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, kcore_peel, kPeelThreads, 0));
    blocks_per_sm = std::max(1, std::min(blocks_per_sm, 2));
    int grid = num_sms() * blocks_per_sm;
    int64_t n_arg = n;
    const int64_t *rp = g->rowptr.get();
    const int32_t *cl = g->col.get();
    int32_t *dg = deg, *co = g->core.get(), *qu = g->peel.get(), *aa = alive_a, *ab = alive_b;
    uint8_t *dd = dead;
    unsigned long long *ct = ctrl;
    void *args[] = {&n_arg, &rp, &cl, &dg, &co, &qu, &aa, &ab, &dd, &ct};
    MCE_CUDA(cudaLaunchCooperativeKernel((void *)kcore_peel, grid, kPeelThreads, args, 0, s));
    g->kernels += 2;
    // degeneracy = max core (the last queued vertex has it)
    last_core_kernel<<<1, 1, 0, s>>>(n, g->peel.get(), g->core.get(), deg);
    int32_t *h = g->host.get<int32_t>(1);
    MCE_CUDA(cudaMemcpyAsync(h, deg, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    MCE_CUDA(cudaStreamSynchronize(s));
    g->degeneracy = h[0];
    g->have_core = true;
}

void orient(mce_graph *g, int orientation) {
    if (g->orientation == orientation) return;
    const int64_t n = g->n;
    cudaStream_t s = g->stream;
    g->order.ensure(std::max<int64_t>(n, 1));
    g->rank.ensure(std::max<int64_t>(n, 1));
    g->orp.ensure(n + 1);
    g->ocol.ensure(std::max<int64_t>(g->nnz / 2, 1));
    g->pool.reset();
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
        int32_t *bins = g->pool.take<int32_t>(nb);
        int64_t *cursor = g->pool.take<int64_t>(nb + 1), *tmp = g->pool.take<int64_t>(scan_tmp_items(nb));
        MCE_CUDA(cudaMemsetAsync(bins, 0, sizeof(int32_t) * nb, s));
        degree_hist<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), bins);
        MCE_LAUNCH_CHECK();
        exclusive_scan_i32(bins, cursor, nb, tmp, s);
        degree_scatter<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), (unsigned long long *)cursor,
                                                         g->order.get());
        MCE_LAUNCH_CHECK();
        g->kernels += 5;
    }
    invert_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->order.get(), g->rank.get());
    MCE_LAUNCH_CHECK();
    int32_t *odeg = g->pool.take<int32_t>(n);
    orient_kernel<false><<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->rowptr.get(), g->col.get(), g->rank.get(), odeg,
                                                               nullptr, nullptr);
    MCE_LAUNCH_CHECK();
    exclusive_scan_i32(odeg, g->orp.get(), n, g->pool.take<int64_t>(scan_tmp_items(n)), s);
    orient_kernel<true><<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->rowptr.get(), g->col.get(), g->rank.get(),
                                                              nullptr, g->orp.get(), g->ocol.get());
    MCE_LAUNCH_CHECK();
    sort_rows_warp<<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->orp.get(), g->ocol.get());
    MCE_LAUNCH_CHECK();
    int32_t *rows = g->pool.take<int32_t>(n), *meta = g->pool.take<int32_t>(2);
    MCE_CUDA(cudaMemsetAsync(meta, 0, 2 * sizeof(int32_t), s));
    long_rows_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->orp.get(), rows, meta, meta + 1);
    MCE_LAUNCH_CHECK();
    int32_t *hmeta = g->host.get<int32_t>(2);
    MCE_CUDA(cudaMemcpyAsync(hmeta, meta, 2 * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    MCE_CUDA(cudaStreamSynchronize(s));
    g->kernels += 8;
    g->max_out = hmeta[1];
    const int32_t n_long = hmeta[0];
    if (n_long > 0) {
        const int32_t smem_cap = 8192;  // ints (32 KB)
        int32_t p2 = 1;
        while (p2 < g->max_out) p2 <<= 1;
        if (p2 <= smem_cap) {
            sort_rows_block<<<grid_for(n_long, 1, 16), 256, smem_cap * sizeof(int32_t), s>>>(
                g->orp.get(), g->ocol.get(), rows, n_long, nullptr, smem_cap);
            MCE_LAUNCH_CHECK();
        } else {  // some row exceeds shared memory: one block, global scratch
            int32_t *scratch = g->pool.take<int32_t>(p2);
            sort_rows_block<<<1, 1024, smem_cap * sizeof(int32_t), s>>>(g->orp.get(), g->ocol.get(), rows, n_long,
                                                                        scratch, smem_cap);
            MCE_LAUNCH_CHECK();
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
