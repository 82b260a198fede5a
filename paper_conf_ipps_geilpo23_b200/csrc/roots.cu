// Root level of the breadth-first search, fused (DESIGN.md §8 row a5, "n1").
//
// PAPER.md IV-C forms the 2-clique list (one sublist per source vertex: its
// out-neighbours under the orientation) and IV-D / Algorithm 2 expands it.
// Here the whole first expansion step of a root r runs inside one warp:
//
//   1. V = N+(r) (|V| = L <= 64) is staged in shared memory (rank order;
//      local index = L-1-position, the reverse degeneracy order of expand.cuh);
//   2. the induced adjacency of V is built by a flattened, warp-cooperative
//      sorted-list intersection: the out-rows N+(v) of every v in V are read
//      32 elements at a time (coalesced within a row), each lane binary-searches
//      its element in the staged V, and a hit (v, u) sets both bits of the
//      L x 64 bit matrix in shared memory;
//   3. the pruning bound of Algorithm 2 line 8 (|C| + |P|, or the colouring
//      bound, reading 5) is evaluated on P = V with rows fetched by
//      __shfl_sync, and the children {r, v} with P' = P-after-v ∩ N(v) are
//      counted (COUNTCLIQUES) and written (OUTPUTNEWCLIQUES) in the same pass;
//   4. only roots with at least one surviving child are materialised: the
//      root record, its adjacency rows and its level-2 entries are appended
//      with one atomicAdd per array (the order of roots inside a level is
//      immaterial: every clique is canonicalised on read-out).
//
// On sparse graphs almost every root is pruned in step 3, so the level-1
// frontier and the adjacency of pruned roots never touch HBM.
#include "expand.cuh"

namespace mce {

namespace {

constexpr int kRootWarps = 8;  // warps per block

struct RootSmem {
    int32_t V[64];
    int32_t off[65];       // flattened row offsets
    int64_t start[64];     // orp[V[i]]
    uint32_t adj[64][2];   // row i, 64 columns as two words
    uint8_t ord[64], colr[64];
    uint8_t chv[64];       // children: local vertex
    uint64_t chP[64];      // children: candidate set
};

__device__ __forceinline__ int lower_bound_smem(const int32_t *a, int n, int32_t key) {
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (a[mid] < key)
            lo = mid + 1;
        else
            hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(kRootWarps * 32) root_expand_w1(const RootArgs a) {
    __shared__ RootSmem sm_all[kRootWarps];
    const int lane = threadIdx.x & 31;
    RootSmem &sm = sm_all[threadIdx.x >> 5];
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long bytes = 0;  // algorithmic bytes read, lane 0
    for (int64_t i = warp; i < a.count; i += nwarps) {
        const int32_t r = __ldg(a.list + i * a.stride);
        const int64_t vb = __ldg(a.orp + r);
        const int L = (int)(__ldg(a.orp + r + 1) - vb);
        // 1. stage V, row starts and lengths
        int len0 = 0, len1 = 0;
        if (lane < L) {
            const int32_t v = __ldg(a.ocol + vb + lane);
            sm.V[lane] = v;
            const int64_t s0 = __ldg(a.orp + v);
            sm.start[lane] = s0;
            len0 = (int)(__ldg(a.orp + v + 1) - s0);
        }
        if (lane + 32 < L) {
            const int32_t v = __ldg(a.ocol + vb + lane + 32);
            sm.V[lane + 32] = v;
            const int64_t s1 = __ldg(a.orp + v);
            sm.start[lane + 32] = s1;
            len1 = (int)(__ldg(a.orp + v + 1) - s1);
        }
        sm.adj[lane][0] = sm.adj[lane][1] = 0u;
        sm.adj[lane + 32][0] = sm.adj[lane + 32][1] = 0u;
        // exclusive offsets of rows 0..63 (row lane, then row lane + 32)
        int inc0 = len0, inc1 = len1;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y0 = __shfl_up_sync(0xffffffffu, inc0, o);
            const int y1 = __shfl_up_sync(0xffffffffu, inc1, o);
            if (lane >= o) {
                inc0 += y0;
                inc1 += y1;
            }
        }
        const int tot0 = __shfl_sync(0xffffffffu, inc0, 31);
        sm.off[lane] = inc0 - len0;
        sm.off[lane + 32] = tot0 + inc1 - len1;
        const int T = tot0 + __shfl_sync(0xffffffffu, inc1, 31);
        if (lane == 0) {
            sm.off[64] = T;
            // root row bounds + V + (row bounds + out-row) of every v in V
            bytes += 16ull + 20ull * (unsigned long long)L + 4ull * (unsigned long long)T;
        }
        __syncwarp();
        // 2. flattened intersection: element t of the concatenated rows
        for (int t0 = 0; t0 < T; t0 += 32) {
            const int t = t0 + lane;
            if (t < T) {
                // row: last i with off[i] <= t (rows past L have length 0 and off == T)
                int lo = 0, hi = L - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (sm.off[mid] <= t)
                        lo = mid;
                    else
                        hi = mid - 1;
                }
                const int32_t u = __ldg(a.ocol + sm.start[lo] + (t - sm.off[lo]));
                const int c = lower_bound_smem(sm.V, L, u);
                if (c < L && sm.V[c] == u) {  // local indices L-1-position (expand.cuh)
                    const int li = L - 1 - lo, lc = L - 1 - c;
                    atomicOr(&sm.adj[li][lc >> 5], 1u << (lc & 31));
                    atomicOr(&sm.adj[lc][li >> 5], 1u << (li & 31));
                }
            }
        }
        __syncwarp();
        const uint64_t row0 = ((uint64_t)sm.adj[lane][1] << 32) | sm.adj[lane][0];
        const uint64_t row1 = ((uint64_t)sm.adj[lane + 32][1] << 32) | sm.adj[lane + 32][0];
        const uint64_t P = L >= 64 ? ~0ull : ((1ull << L) - 1);
        // 3. bound + children (|C| = 1)
        int np = 0, ncol = 0;
        if (a.bound == 1) {
            uint64_t U = P;
            while (U) {
                ++ncol;
                uint64_t Q = U;
                while (Q) {
                    const int v = __ffsll((long long)Q) - 1;
                    const uint64_t rv0 = __shfl_sync(0xffffffffu, row0, v & 31);
                    const uint64_t rv1 = __shfl_sync(0xffffffffu, row1, v & 31);
                    const uint64_t rv = v < 32 ? rv0 : rv1;
                    Q &= ~rv;
                    Q &= ~(1ull << v);
                    U &= ~(1ull << v);
                    if (lane == 0) {
                        sm.ord[np] = (uint8_t)v;
                        sm.colr[np] = (uint8_t)ncol;
                    }
                    ++np;
                }
            }
        } else {
            if (lane == 0)
                for (int j = 0; j < L; ++j) {
                    sm.ord[j] = (uint8_t)j;
                    sm.colr[j] = (uint8_t)(j + 1);
                }
            np = ncol = L;
        }
        __syncwarp();
        int cnt = 0;
        if (1 + ncol >= a.need) {
            uint64_t R = P;
            for (int j = np - 1; j >= 0; --j) {
                if (1 + sm.colr[j] < a.need) break;
                const int v = sm.ord[j];
                const uint64_t rv0 = __shfl_sync(0xffffffffu, row0, v & 31);
                const uint64_t rv1 = __shfl_sync(0xffffffffu, row1, v & 31);
                const uint64_t C = R & (v < 32 ? rv0 : rv1);
                R &= ~(1ull << v);
                const int pc = __popcll(C);
                if (pc == 0) {
                    if (2 >= a.need && lane == 0) {  // {r, v} is a leaf clique of interest
                        const unsigned long long idx = atomicAdd(a.ctr + 3, 1ull);
                        if ((int64_t)idx < a.leaf_cap) {
                            a.leaf_rows[idx * 2] = __ldg(a.order + r);
                            a.leaf_rows[idx * 2 + 1] = __ldg(a.order + sm.V[L - 1 - v]);
                        }
                    }
                } else if (2 + pc >= a.need) {
                    if (lane == 0) {
                        sm.chv[cnt] = (uint8_t)v;
                        sm.chP[cnt] = C;
                    }
                    ++cnt;
                }
            }
        }
        // 4. materialise surviving roots
        if (cnt > 0) {
            unsigned long long s = 0, ab = 0, e0 = 0;
            if (lane == 0) {
                s = atomicAdd(a.ctr + 0, 1ull);
                ab = atomicAdd(a.ctr + 1, (unsigned long long)L);
                e0 = atomicAdd(a.ctr + 2, (unsigned long long)cnt);
            }
            s = __shfl_sync(0xffffffffu, s, 0);
            ab = __shfl_sync(0xffffffffu, ab, 0);
            e0 = __shfl_sync(0xffffffffu, e0, 0);
            __syncwarp();
            if (lane == 0) {
                RootInfo ri;
                ri.r = r;
                ri.L = L;
                ri.vbase = vb;
                ri.abase = (int64_t)ab;
                a.roots[s] = ri;
            }
            if (lane < L) a.adj[ab + lane] = row0;
            if (lane + 32 < L) a.adj[ab + lane + 32] = row1;
            for (int j = lane; j < cnt; j += 32) {
                a.cP[e0 + j] = sm.chP[j];
                a.cslot[e0 + j] = (int32_t)s;
                a.cparent[e0 + j] = -1;
                a.cvloc[e0 + j] = sm.chv[j];
            }
        }
        __syncwarp();
    }
    if (lane == 0 && bytes) atomicAdd(a.ctr + 4, bytes);
}

}  // namespace

void launch_root_expand_w1(const RootArgs &a, cudaStream_t s) {
    if (a.count <= 0) return;
    root_expand_w1<<<grid_for(a.count * 32, kRootWarps * 32, 8), kRootWarps * 32, 0, s>>>(a);
    MCE_LAUNCH_CHECK();
}

}  // namespace mce
