// Root colour filter (reading 14): drop roots whose out-neighbourhood
// cannot hold a clique of the size sought, before their adjacency matrix is
// built.
//
// Every vertex of a clique of size s has core number >= s - 1 (the clique is
// itself an (s-1)-core subgraph; PAPER.md II-B-2, line 61), so only the set
//   S = { v : core(v) >= need - 1 }
// matters, and under a degeneracy orientation S is both the top |S| ranks
// (the peel order is non-decreasing in core) and the suffix [T, n) of CSR-id
// space (ids are sorted by core).  S is coloured greedily in reverse
// degeneracy order (smallest-last, Matula-Beck): vertex v takes the smallest
// colour not used by its out-neighbours N+(v), which are exactly the
// neighbours coloured before it.  Any proper colouring of G restricted to
// N+(r) bounds every clique inside it, so a root r with
//   1 + |colours(N+(r))| < need
// has no clique of size need (the colouring bound of PAPER.md II-B-3, line 63,
// taken from a global colouring instead of the root's own) and is dropped.
//
// The greedy colouring is sequential in the order; on the device it runs as
// a dataflow: persistent warps take vertices in order (one atomic counter),
// wait for the colours of their out-neighbours (all taken earlier, by running
// warps, so the wait always ends), and publish their own.  The critical path is
// the longest chain of the orientation DAG inside S (2581 vertices on rmat22,
// whose 35.5K-vertex S prunes 27K of its 35K roots of out-degree >= 222).
#include <cooperative_groups.h>

#include "graph.cuh"

namespace mce {

namespace {

__device__ __forceinline__ int32_t ld_relaxed_i32(const int32_t *p) {
    int32_t v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_i32(int32_t *p, int32_t v) {
    asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// T = the first CSR id whose core number is >= c (core by CSR id is non-decreasing)
__global__ void core_threshold_kernel(int64_t n, const int32_t *__restrict__ vid, const int32_t *__restrict__ core,
                                      int32_t c, int64_t *out) {
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (core[vid[mid]] < c)
            lo = mid + 1;
        else
            hi = mid;
    }
    out[0] = lo;
}

constexpr int kColWarps = 8;  // warps per block of both kernels
#ifndef COL_CLUSTER
#define COL_CLUSTER 1  // S small enough for shared memory: colour inside one 8-CTA cluster (DSMEM)
#endif
#ifndef COL_BACKOFF
#define COL_BACKOFF 1  // poll back-off by the number of colours still missing (0: fixed 32 / 128 ns)
#endif
#ifndef COL_SPIN
#define COL_SPIN 0  // polls of the pending list before the first back-off sleep
#endif

// greedy colouring of the top m ranks (= CSR ids [T, n)), colr[id - T].
// Per vertex: one pass over its out-row with independent loads ORs every
// colour already published into the warp's mask and lists the out-neighbours
// still uncoloured (shared memory); only that list is polled afterwards, so a
// vertex finishes about one L2 round trip after its last predecessor (the
// critical path is one such step per vertex of the longest chain).
__global__ void __launch_bounds__(32 * kColWarps) colour_dataflow_kernel(
    int64_t n, int64_t m, int64_t T, const int32_t *__restrict__ order, const int32_t *__restrict__ pid,
    const int64_t *__restrict__ orp, const int32_t *__restrict__ ocol, int MW, int PW, int32_t *colr,
    unsigned long long *next) {
    extern __shared__ unsigned smask_all[];
    const int lane = threadIdx.x & 31;
    unsigned *mask = smask_all + (size_t)(threadIdx.x >> 5) * (MW + PW);
    int32_t *pend = reinterpret_cast<int32_t *>(mask + MW);
    while (true) {
        unsigned long long j = 0;
        if (lane == 0) j = atomicAdd(next, 1ull);
        j = __shfl_sync(0xffffffffu, j, 0);
        if ((int64_t)j >= m) break;
        const int32_t i = pid[order[n - 1 - (int64_t)j]];
        const int64_t rb = orp[i], re = orp[i + 1];
        for (int w = lane; w < MW; w += 32) mask[w] = 0u;
        __syncwarp();
        int np = 0;  // pending entries (warp-uniform)
        for (int64_t e0 = rb; e0 < re; e0 += 256) {
            int32_t u[8], c[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const int64_t e = e0 + 32 * q + lane;
                u[q] = e < re ? __ldg(ocol + e) : -1;
            }
#pragma unroll
            for (int q = 0; q < 8; ++q) c[q] = u[q] >= 0 ? ld_relaxed_i32(colr + (u[q] - T)) : -2;
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                if (c[q] >= 0) atomicOr(mask + (c[q] >> 5), 1u << (c[q] & 31));
                const unsigned pm = __ballot_sync(0xffffffffu, c[q] == -1);
                if (c[q] == -1) pend[np + __popc(pm & lanemask_lt())] = u[q];
                np += __popc(pm);
            }
        }
        int naps = 0;
        while (np > 0) {  // poll the uncoloured out-neighbours (taken by running warps: the wait ends)
            __syncwarp();
            int left = 0;
            for (int b = 0; b < np; b += 32) {
                const int t = b + lane;
                int32_t u = -1, c = -2;
                if (t < np) {
                    u = pend[t];
                    c = ld_relaxed_i32(colr + (u - T));
                }
                if (c >= 0) atomicOr(mask + (c >> 5), 1u << (c & 31));
                const unsigned pm = __ballot_sync(0xffffffffu, c == -1);
                __syncwarp();
                if (c == -1) pend[left + __popc(pm & lanemask_lt())] = u;  // left <= b: no overwrite of unread entries
                left += __popc(pm);
            }
            np = left;
            if (np > 0) {
                // back off in proportion to how much is still missing: a warp waiting
                // for many predecessors is far from the chain's head, and thousands of
                // warps polling at full rate load the L2 the chain's own loads and
                // stores go through
                if (COL_BACKOFF)
                    __nanosleep(np > 16 ? 2048 : (np > 4 ? 512 : (np > 1 ? 128 : 32)));
                else if (naps >= COL_SPIN)
                    __nanosleep(naps < COL_SPIN + 8 ? 32 : 128);
                ++naps;
            }
        }
        __syncwarp();
        int first = INT32_MAX;
        for (int w = lane; w < MW; w += 32) {
            const unsigned z = ~mask[w];
            if (z) {
                first = w * 32 + __ffs((int)z) - 1;
                break;  // words are visited in increasing order per lane
            }
        }
        first = __reduce_min_sync(0xffffffffu, first);
        if (lane == 0) st_relaxed_i32(colr + (i - T), first);
        __syncwarp();
    }
}

// The same greedy colouring inside ONE thread-block cluster (kClusterCtas SMs)
// when S is small enough for every CTA to hold all of S's colours (u16) in
// its shared memory: a published colour is written into every CTA's copy
// through distributed shared memory (st to cluster.map_shared_rank: ~200
// cycles, not an L2 round trip), and a waiting warp polls its own CTA's copy.
// A step of the critical chain then costs one DSMEM store plus a shared-memory
// poll instead of an L2 store plus an L2 poll (rmat22: 2581 steps).  Vertices
// are taken in order from a counter in CTA 0's shared memory; every warp of
// the cluster is resident, so a waited-for vertex is always being coloured.
constexpr int kClusterCtas = 8;        // portable cluster size
constexpr int kClusterWarps = 32;      // warps per CTA
#ifndef COL_PEND
#define COL_PEND 12
#endif
constexpr int kClusterPend = COL_PEND;  // pending predecessors a lane keeps (shared memory); measured 4 / 12 / 24 = 4.7 / 2.4 / 2.4 ms on rmat22
constexpr uint16_t kNoColour = 0xffffu;

__global__ void __launch_bounds__(32 * kClusterWarps) colour_cluster_kernel(
    int64_t n, int64_t m, int64_t T, const int32_t *__restrict__ order, const int32_t *__restrict__ pid,
    const int64_t *__restrict__ orp, const int32_t *__restrict__ ocol, int MW, int32_t *colr) {
    namespace cg = cooperative_groups;
    cg::cluster_group cluster = cg::this_cluster();
    extern __shared__ unsigned char csm[];
    unsigned long long *next = reinterpret_cast<unsigned long long *>(csm);           // (CTA 0's is used)
    int32_t *pends = reinterpret_cast<int32_t *>(csm + 16);                            // threads x kClusterPend
    unsigned *masks = reinterpret_cast<unsigned *>(pends + (size_t)32 * kClusterWarps * kClusterPend);
    uint16_t *scol = reinterpret_cast<uint16_t *>(masks + (size_t)kClusterWarps * MW);  // m colours
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    unsigned *mask = masks + (size_t)wib * MW;
    int32_t *pend = pends + (size_t)threadIdx.x * kClusterPend;  // this lane's pending predecessors
    for (int64_t j = threadIdx.x; j < m; j += blockDim.x) scol[j] = kNoColour;
    if (threadIdx.x == 0) *next = 0ull;
    cluster.sync();
    unsigned long long *gnext = cluster.map_shared_rank(next, 0);
    while (true) {
        unsigned long long j = 0;
        if (lane == 0) j = atomicAdd(gnext, 1ull);
        j = __shfl_sync(0xffffffffu, j, 0);
        if ((int64_t)j >= m) break;
        const int32_t i = pid[order[n - 1 - (int64_t)j]];
        const int64_t rb = orp[i], re = orp[i + 1];
        for (int w = lane; w < MW; w += 32) mask[w] = 0u;
        __syncwarp();
        int np = 0;
        bool rescan = false;  // more than kClusterPend pending in this lane's elements
        // the row's ids are loaded 8 per lane at a time, all in flight together (a
        // dense-core row of ~1000 ids is then a few L2 latencies, not ~30)
        for (int64_t e0 = rb; e0 < re; e0 += 32 * 8) {
            int32_t uu[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const int64_t e = e0 + 32 * q + lane;
                uu[q] = e < re ? __ldg(ocol + e) - (int32_t)T : -1;
            }
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                if (uu[q] < 0) continue;
                const uint16_t c = *(volatile uint16_t *)(scol + uu[q]);
                if (c != kNoColour) {
                    atomicOr(mask + (c >> 5), 1u << (c & 31));
                } else if (np < kClusterPend) {
                    pend[np++] = uu[q];
                } else {
                    rescan = true;
                }
            }
        }
        // wait for the missing colours (predecessors are taken earlier by resident warps)
        while (__any_sync(0xffffffffu, np > 0 || rescan)) {
            int left = 0;
            for (int q = 0; q < np; ++q) {
                const int32_t u = pend[q];
                const uint16_t c = *(volatile uint16_t *)(scol + u);
                if (c != kNoColour)
                    atomicOr(mask + (c >> 5), 1u << (c & 31));
                else
                    pend[left++] = u;
            }
            np = left;
            if (rescan && np == 0) {  // re-read this lane's elements for the overflowed ones
                rescan = false;
                for (int64_t e0 = rb; e0 < re; e0 += 32 * 8) {
                    int32_t uu[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        const int64_t e = e0 + 32 * q + lane;
                        uu[q] = e < re ? __ldg(ocol + e) - (int32_t)T : -1;
                    }
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        if (uu[q] < 0) continue;
                        const uint16_t c = *(volatile uint16_t *)(scol + uu[q]);
                        if (c != kNoColour)
                            atomicOr(mask + (c >> 5), 1u << (c & 31));  // (idempotent)
                        else if (np < kClusterPend)
                            pend[np++] = uu[q];
                        else
                            rescan = true;
                    }
                }
            }
            if (np > 0 || rescan) __nanosleep(20);
        }
        __syncwarp();
        int first = INT32_MAX;
        for (int w = lane; w < MW; w += 32) {
            const unsigned z = ~mask[w];
            if (z) {
                first = w * 32 + __ffs((int)z) - 1;
                break;
            }
        }
        first = __reduce_min_sync(0xffffffffu, first);
        if (lane < kClusterCtas)  // every CTA's copy, through distributed shared memory
            *(volatile uint16_t *)cluster.map_shared_rank(scol + (i - T), lane) = (uint16_t)first;
        if (lane == 0) colr[i - T] = first;
        __syncwarp();
    }
    cluster.sync();  // no CTA leaves while others may still write into its shared memory
}

// keep[r - T] = 1 + |colours(N+(r))| >= need (and |N+(r)| >= need - 1), warp per root
__global__ void __launch_bounds__(32 * kColWarps) root_colour_bound_kernel(
    int64_t n, int64_t T, const int64_t *__restrict__ orp, const int32_t *__restrict__ ocol,
    const int32_t *__restrict__ colr, int MW, int32_t need, uint8_t *keep, unsigned long long *kept) {
    extern __shared__ unsigned smask_all[];
    const int lane = threadIdx.x & 31;
    unsigned *mask = smask_all + (size_t)(threadIdx.x >> 5) * MW;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long mine = 0;
    for (int64_t r = T + warp; r < n; r += nwarps) {
        const int64_t rb = orp[r], re = orp[r + 1];
        bool ok = false;
        if (re - rb >= need - 1) {
            for (int w = lane; w < MW; w += 32) mask[w] = 0u;
            __syncwarp();
            for (int64_t e = rb + lane; e < re; e += 32) {
                const int32_t c = __ldg(colr + (__ldg(ocol + e) - T));
                atomicOr(mask + (c >> 5), 1u << (c & 31));
            }
            __syncwarp();
            int cnt = 0;
            for (int w = lane; w < MW; w += 32) cnt += __popc(mask[w]);
            cnt = __reduce_add_sync(0xffffffffu, cnt);
            ok = cnt + 1 >= need;
            __syncwarp();
        }
        if (lane == 0) {
            keep[r - T] = ok ? 1 : 0;
            mine += ok;
        }
    }
    if (lane == 0 && mine) atomicAdd(kept, mine);
}

}  // namespace

// Runs the filter when it can pay: a degeneracy orientation (S is a rank
// suffix), at least min_s vertices in S, and out-degrees below 2^12.  On
// success keep (m = n - T bytes, caller-provided, at least n) holds the
// flags of CSR ids [T, n) and the function returns true with *T_out, *kept_out.
// (the dataflow kernel holds a colour mask and a pending list
// of max_out + 1 entries per warp in shared memory)
bool root_colour_filter(mce_graph *g, int32_t need, int64_t min_s, uint8_t *keep, int32_t *colr, int64_t *scratch,
                        cudaStream_t s, int64_t *T_out, int64_t *kept_out) {
    const int64_t n = g->n;
    if (n == 0 || need < 3 || (g->orientation != 0 && g->orientation != 2) || g->max_out >= (1 << 12)) return false;
    core_threshold_kernel<<<1, 1, 0, s>>>(n, g->vid.get(), g->core.get(), need - 1, scratch);
    MCE_LAUNCH_CHECK();
    int64_t *h = g->host.get<int64_t>(1);
    MCE_CUDA(cudaMemcpyAsync(h, scratch, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    stream_sync(s);
    const int64_t T = h[0], m = n - T;
    if (m < min_s) return false;
    const int MW = (g->max_out + 1 + 31) / 32;           // colour mask words (colours <= out-degree)
    const int PW = (g->max_out + 3) & ~3;                  // pending list of one vertex
    const size_t smem = (size_t)kColWarps * MW * sizeof(unsigned);
    const size_t smem_df = (size_t)kColWarps * (MW + PW) * sizeof(unsigned);
    unsigned long long *ctr = reinterpret_cast<unsigned long long *>(scratch + 1);  // [0] next, [1] kept
    MCE_CUDA(cudaMemsetAsync(ctr, 0, 2 * sizeof(unsigned long long), s));
    MCE_CUDA(cudaMemsetAsync(colr, 0xff, sizeof(int32_t) * m, s));
    if (smem_df > 48 * 1024)
        MCE_CUDA(cudaFuncSetAttribute(colour_dataflow_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_df));
    if (smem > 48 * 1024)
        MCE_CUDA(cudaFuncSetAttribute(root_colour_bound_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const size_t csmem = 16 + (size_t)32 * kClusterWarps * kClusterPend * 4 + (size_t)kClusterWarps * MW * 4 +
                         (size_t)m * 2;
    if (COL_CLUSTER && csmem <= 200 * 1024 && MW <= 64) {
        static size_t attr = 0;
        if (attr < csmem) {
            MCE_CUDA(cudaFuncSetAttribute(colour_cluster_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)csmem));
            attr = csmem;
        }
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(kClusterCtas, 1, 1);
        cfg.blockDim = dim3(32 * kClusterWarps, 1, 1);
        cfg.dynamicSmemBytes = csmem;
        cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = kClusterCtas;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        const int32_t *ord = g->order.get(), *pd = g->pid.get(), *oc = g->ocol.get();
        const int64_t *op = g->orp.get();
        MCE_CUDA(cudaLaunchKernelEx(&cfg, colour_cluster_kernel, n, m, T, ord, pd, op, oc, MW, colr));
    } else {
    // persistent dataflow: only resident warps may take vertices (a waiting
    // warp's predecessors must be running), so the grid is the resident capacity
    int per_sm = 0;
    MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, colour_dataflow_kernel, 32 * kColWarps, smem_df));
    if (per_sm < 1) return false;
    const int grid = (int)std::min<int64_t>((int64_t)num_sms() * per_sm, (m + kColWarps - 1) / kColWarps);
    colour_dataflow_kernel<<<grid, 32 * kColWarps, smem_df, s>>>(n, m, T, g->order.get(), g->pid.get(), g->orp.get(),
                                                                 g->ocol.get(), MW, PW, colr, ctr);
    MCE_LAUNCH_CHECK();
    }
    root_colour_bound_kernel<<<grid_for(m * 32, 32 * kColWarps, 8), 32 * kColWarps, smem, s>>>(
        n, T, g->orp.get(), g->ocol.get(), colr, MW, need, keep, ctr + 1);
    MCE_LAUNCH_CHECK();
    unsigned long long *hk = g->host.get<unsigned long long>(1);
    MCE_CUDA(cudaMemcpyAsync(hk, ctr + 1, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    stream_sync(s);
    *T_out = T;
    *kept_out = (int64_t)hk[0];
    return true;
}

}  // namespace mce
