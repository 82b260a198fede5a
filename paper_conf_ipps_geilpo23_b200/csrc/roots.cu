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
#include <type_traits>
#include "expand.cuh"

namespace mce {

namespace {

constexpr int kRootWarps = 8;  // warps per block

// per-tile scratch for one root of up to M = G * RPL candidates
template <int M>
struct RootSmem {
    int32_t V[M];
    int32_t off[M + 1];    // flattened row offsets
    int64_t start[M];      // orp[V[i]]
    uint32_t adj[M][2];    // row of local index i, 64 columns as two words
    uint8_t ord[M], colr[M];
    uint8_t chv[M];        // children: local vertex
    uint64_t chP[M];       // children: candidate set
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

// The whole first expansion step of root r (|N+(r)| = L <= G * RPL) by a tile
// of G lanes; lane gl owns local rows gl, gl + G, ... (RPL of them).
template <int G, int RPL>
__device__ void root_step(const RootArgs &a, int32_t r, RootSmem<G * RPL> &sm, unsigned long long &bytes) {
    constexpr int M = G * RPL;
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1), gbase = lane & ~(G - 1);
    const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
    const int64_t vb = __ldg(a.orp + r);
    const int L = (int)(__ldg(a.orp + r + 1) - vb);
    // 1. stage V (rank order), row starts and lengths; zero the bit matrix
    int len[RPL];
#pragma unroll
    for (int q = 0; q < RPL; ++q) {
        const int p = gl + q * G;
        len[q] = 0;
        if (p < L) {
            const int32_t v = __ldg(a.ocol + vb + p);
            sm.V[p] = v;
            const int64_t s0 = __ldg(a.orp + v);
            sm.start[p] = s0;
            len[q] = (int)(__ldg(a.orp + v + 1) - s0);
        }
        sm.adj[p][0] = sm.adj[p][1] = 0u;
    }
    // exclusive offsets of rows 0..M-1 in position order
    int carry = 0;
#pragma unroll
    for (int q = 0; q < RPL; ++q) {
        int inc = len[q];
#pragma unroll
        for (int o = 1; o < G; o <<= 1) {
            const int y = __shfl_up_sync(gmask, inc, o, G);
            if (gl >= o) inc += y;
        }
        sm.off[gl + q * G] = carry + inc - len[q];
        carry += __shfl_sync(gmask, inc, G - 1, G);
    }
    const int T = carry;
    if (gl == 0) {
        sm.off[M] = T;
        // root row bounds + V + (row bounds + out-row) of every v in V
        bytes += 16ull + 20ull * (unsigned long long)L + 4ull * (unsigned long long)T;
    }
    __syncwarp(gmask);
    // 2. flattened intersection: element t of the concatenated out-rows
    for (int t0 = 0; t0 < T; t0 += G) {
        const int t = t0 + gl;
        if (t < T) {
            int lo = 0, hi = L - 1;  // row: last i with off[i] <= t
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
    __syncwarp(gmask);
    uint64_t row[RPL];
#pragma unroll
    for (int q = 0; q < RPL; ++q) {
        const int p = gl + q * G;
        row[q] = ((uint64_t)sm.adj[p][1] << 32) | sm.adj[p][0];
    }
    const uint64_t P = L >= 64 ? ~0ull : ((1ull << L) - 1);
    auto fetch = [&](int v) -> uint64_t {  // row of local v, from the lane that owns it
        uint64_t x = 0;
#pragma unroll
        for (int q = 0; q < RPL; ++q) {
            const uint64_t y = __shfl_sync(gmask, row[q], v & (G - 1), G);
            if (v / G == q) x = y;
        }
        return x;
    };
    // 3. bound + children (|C| = 1)
    int np = 0, ncol = 0;
    if (a.bound == 1) {
        uint64_t U = P;
        while (U) {
            ++ncol;
            uint64_t Q = U;
            while (Q) {
                const int v = __ffsll((long long)Q) - 1;
                Q &= ~fetch(v);
                Q &= ~(1ull << v);
                U &= ~(1ull << v);
                if (gl == 0) {
                    sm.ord[np] = (uint8_t)v;
                    sm.colr[np] = (uint8_t)ncol;
                }
                ++np;
            }
        }
    } else {
        if (gl == 0)
            for (int j = 0; j < L; ++j) {
                sm.ord[j] = (uint8_t)j;
                sm.colr[j] = (uint8_t)(j + 1);
            }
        np = ncol = L;
    }
    __syncwarp(gmask);
    int cnt = 0;
    if (1 + ncol >= a.need) {
        uint64_t R = P;
        for (int j = np - 1; j >= 0; --j) {
            if (1 + sm.colr[j] < a.need) break;
            const int v = sm.ord[j];
            const uint64_t C = R & fetch(v);
            R &= ~(1ull << v);
            const int pc = __popcll(C);
            if (pc == 0) {
                if (2 >= a.need && gl == 0) {  // {r, v} is a leaf clique of interest
                    const unsigned long long idx = atomicAdd(a.ctr + 3, 1ull);
                    if ((int64_t)idx < a.leaf_cap) {
                        a.leaf_rows[idx * 2] = __ldg(a.order + r);
                        a.leaf_rows[idx * 2 + 1] = __ldg(a.order + sm.V[L - 1 - v]);
                    }
                }
            } else if (2 + pc >= a.need) {
                if (gl == 0) {
                    sm.chv[cnt] = (uint8_t)v;
                    sm.chP[cnt] = C;
                }
                ++cnt;
            }
        }
    }
    // 4. materialise a surviving root: record, adjacency rows, level-2 entries
    if (cnt > 0) {
        unsigned long long s = 0, ab = 0, e0 = 0;
        if (gl == 0) {
            s = atomicAdd(a.ctr + 0, 1ull);
            ab = atomicAdd(a.ctr + 1, (unsigned long long)L);
            e0 = atomicAdd(a.ctr + 2, (unsigned long long)cnt);
        }
        s = __shfl_sync(gmask, s, 0, G);
        ab = __shfl_sync(gmask, ab, 0, G);
        e0 = __shfl_sync(gmask, e0, 0, G);
        __syncwarp(gmask);
        if (gl == 0) {
            RootInfo ri;
            ri.r = r;
            ri.L = L;
            ri.vbase = vb;
            ri.abase = (int64_t)ab;
            a.roots[s] = ri;
        }
#pragma unroll
        for (int q = 0; q < RPL; ++q)
            if (gl + q * G < L) a.adj[ab + gl + q * G] = row[q];
        for (int j = gl; j < cnt; j += G) {
            a.cP[e0 + j] = sm.chP[j];
            a.cslot[e0 + j] = (int32_t)s;
            a.cparent[e0 + j] = -1;
            a.cvloc[e0 + j] = sm.chv[j];
        }
    }
    __syncwarp(gmask);
}

// 8x8 bit-matrix transpose (row i = byte i, column j = bit j)
__device__ __forceinline__ uint64_t transpose8(uint64_t x) {
    uint64_t t;
    t = (x ^ (x >> 7)) & 0x00AA00AA00AA00AAull;
    x = x ^ t ^ (t << 7);
    t = (x ^ (x >> 14)) & 0x0000CCCC0000CCCCull;
    x = x ^ t ^ (t << 14);
    t = (x ^ (x >> 28)) & 0x00000000F0F0F0F0ull;
    x = x ^ t ^ (t << 28);
    return x;
}

// warp exclusive prefix sum of x (all 32 lanes; per-lane values and the warp
// total fit 32 bits: at most 32 roots x 64 rows or children)
__device__ __forceinline__ unsigned warp_excl(unsigned x, unsigned &total) {
    const int lane = threadIdx.x & 31;
    unsigned inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    total = __shfl_sync(0xffffffffu, inc, 31);
    return inc - x;
}

// The whole first expansion step of a root with L = |N+(r)| <= 8 by ONE
// thread (the sparse case: BA m = 4 roots have L = 4).  Same steps as
// root_step, in registers: the L x L bit matrix is one uint64 (row li = byte
// li), built by testing every element of each out-row N+(V[p]) against the
// L staged ids (or, for a long out-row, binary-searching the L ids in it) and
// closed under symmetry with an 8x8 transpose; the colouring order, colours
// and children are packed nibbles / bytes.  Called by all 32 lanes of a warp
// (r < 0: no root) so survivors are materialised with warp-aggregated atomics.
// Thread-per-root loads are scattered (every lane its own line), so the L1
// wavefronts they cost, not bytes, bound the root level (ncu: LSU data-pipe
// wavefronts 77% of peak).  These helpers fetch what one lane needs with
// aligned 16-byte loads: a row's bounds orp[v], orp[v+1] in one load when v is
// even, up to four consecutive ids in one or two.
__device__ __forceinline__ void row_bounds(const int64_t *__restrict__ orp, int32_t v, int64_t &b, int64_t &e) {
    const longlong2 x = __ldg(reinterpret_cast<const longlong2 *>(orp + (v & ~1)));
    if (v & 1) {
        b = x.y;
        e = __ldg(orp + v + 1);
    } else {
        b = x.x;
        e = x.y;
    }
}

// u[k] = col[s + k] for k < d (d <= 4), else fill.  The int4 loads may read up
// to three ids past the end of `col` (the oriented CSR is allocated with that
// padding, preprocess.cu).
__device__ __forceinline__ void load4(const int32_t *__restrict__ col, int64_t s, int d, int32_t fill,
                                      int32_t (&u)[4]) {
    const int64_t al = s & ~3ll;
    const int o = (int)(s - al);
    int4 w0 = make_int4(fill, fill, fill, fill), w1 = w0;
    if (d > 0) w0 = __ldg(reinterpret_cast<const int4 *>(col + al));
    if (o + d > 4) w1 = __ldg(reinterpret_cast<const int4 *>(col + al + 4));
    const int32_t x[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
    int32_t y[6];
#pragma unroll
    for (int i = 0; i < 6; ++i) y[i] = (o & 2) ? x[i + 2] : x[i];
#pragma unroll
    for (int k = 0; k < 4; ++k) u[k] = k < d ? ((o & 1) ? y[k + 1] : y[k]) : fill;
}

// kShort: every out-row of the launch has <= 4 ids (the orientation's largest
// out-degree is <= 4), so the tail and binary-search paths are compiled out
// kPad: the rows come from the 16-byte padded copy (a.ocol4; kShort only):
// a root's row and each neighbour's row are one aligned load each, with no
// row bounds (vb and L are derived here; vb is read only for survivors)
template <int LM, bool kShort = false, bool kPad = false>
__device__ void root_thread(const RootArgs &a, int32_t r, int64_t vb, int L, unsigned long long &bytes) {
    static_assert(!kPad || (kShort && LM == 4), "padded rows: sparse launches only");
    uint64_t adj = 0;
    typename std::conditional<kShort, unsigned, unsigned long long>::type T = 0;
    int32_t V[LM];
    if (r < 0) {
        vb = 0;
        L = 0;
    }
    if (kPad && r >= 0) {
        const int4 x = __ldg(a.ocol4 + r);
        V[0] = x.x;
        V[1] = x.y;
        V[2] = x.z;
        V[3] = x.w;
        L = (x.x >= 0) + (x.y >= 0) + (x.z >= 0) + (x.w >= 0);
        int4 y[4];
#pragma unroll
        for (int p = 0; p < 4; ++p) y[p] = p < L ? __ldg(a.ocol4 + V[p]) : make_int4(-2, -2, -2, -2);
#pragma unroll
        for (int p = 0; p < 4; ++p) {
            if (p >= L) break;
            const int32_t u0 = y[p].x, u1 = y[p].y, u2 = y[p].z, u3 = y[p].w;
            T += (u0 >= 0) + (u1 >= 0) + (u2 >= 0) + (u3 >= 0);
            unsigned m = 0;
#pragma unroll
            for (int c = 0; c < 4; ++c)
                m |= (unsigned)((V[c] == u0) | (V[c] == u1) | (V[c] == u2) | (V[c] == u3)) << c;
            const unsigned lm = (__brev(m) >> (32 - L)) & 0xffu;
            adj |= (uint64_t)lm << (8 * (L - 1 - p));
        }
        adj |= transpose8(adj);
        // the method's bytes over the CSR, as for the unpadded path
        bytes += 16ull + 20ull * (unsigned long long)L + 4ull * T;
    }
    if (!kPad && r >= 0) {
        if constexpr (LM == 4) {
            load4(a.ocol, vb, L, -1, V);
        } else {
#pragma unroll
            for (int p = 0; p < LM; ++p) V[p] = p < L ? __ldg(a.ocol + vb + p) : -1;
        }
        // kShort launches also guarantee |E+| < 2^31 (engine.cu): 32-bit offsets
        using Off = typename std::conditional<kShort, int32_t, int64_t>::type;
        Off s0[LM], s1[LM];
#pragma unroll
        for (int p = 0; p < LM; ++p) {
            s0[p] = s1[p] = 0;
            if (p < L) {
                int64_t b, e;
                row_bounds(a.orp, V[p], b, e);
                s0[p] = (Off)b;
                s1[p] = (Off)e;
            }
        }
        // LM == 4 (sparse roots): the first four elements of every out-row,
        // all issued before any is used, so the adjacency costs one load
        // latency, not one per row
        int32_t u[LM == 4 ? 4 : 1][4];
        if constexpr (LM == 4) {
#pragma unroll
            for (int p = 0; p < 4; ++p) {
                const Off d = s1[p] - s0[p];
                load4(a.ocol, s0[p], (p < L && (kShort || d <= 16)) ? (int)min(d, (Off)4) : 0, -2, u[p]);
            }
        }
#pragma unroll
        for (int p = 0; p < LM; ++p) {
            if (p >= L) break;
            const int64_t d = s1[p] - s0[p];
            T += d;
            unsigned m = 0;  // positions c with V[c] in N+(V[p])
            if (kShort || d <= 16) {
                // the first four elements as independent loads (sparse out-rows are
                // that short), so a row costs one load latency, not d of them
                int32_t u0, u1, u2, u3;
                if constexpr (LM == 4) {
                    u0 = u[p][0];
                    u1 = u[p][1];
                    u2 = u[p][2];
                    u3 = u[p][3];
                } else {
                    u0 = d > 0 ? __ldg(a.ocol + s0[p]) : -2;
                    u1 = d > 1 ? __ldg(a.ocol + s0[p] + 1) : -2;
                    u2 = d > 2 ? __ldg(a.ocol + s0[p] + 2) : -2;
                    u3 = d > 3 ? __ldg(a.ocol + s0[p] + 3) : -2;
                }
#pragma unroll
                for (int c = 0; c < LM; ++c)
                    m |= (unsigned)((V[c] == u0) | (V[c] == u1) | (V[c] == u2) | (V[c] == u3)) << c;
                if constexpr (!kShort) {
                    for (int64_t q = s0[p] + 4; q < s1[p]; ++q) {
                        const int32_t u = __ldg(a.ocol + q);
#pragma unroll
                        for (int c = 0; c < LM; ++c) m |= (unsigned)(V[c] == u) << c;
                    }
                }
            } else {
#pragma unroll
                for (int c = 0; c < LM; ++c)
                    if (c < L && c != p && contains_sorted(a.ocol, s0[p], s1[p], V[c])) m |= 1u << c;
            }
            // local index = L-1-position (expand.cuh): reverse rows and columns
            const unsigned lm = (__brev(m) >> (32 - L)) & 0xffu;
            adj |= (uint64_t)lm << (8 * (L - 1 - p));
        }
        adj |= transpose8(adj);
        bytes += 16ull + 20ull * (unsigned long long)L + 4ull * T;
    }
    auto row = [&](int v) -> uint64_t { return (adj >> (8 * v)) & 0xffull; };
    // bound + children (|C| = 1)
    const uint64_t P = (1ull << L) - 1;
    uint32_t ord = 0, colr = 0;  // nibble j: j-th vertex in colouring order, its colour
    int np = 0, ncol = 0;
    if (a.bound == 1) {
        uint64_t U = P;
        while (U) {
            ++ncol;
            uint64_t Q = U;
            while (Q) {
                const int v = __ffsll((long long)Q) - 1;
                Q &= ~row(v);
                Q &= ~(1ull << v);
                U &= ~(1ull << v);
                ord |= (uint32_t)v << (4 * np);
                colr |= (uint32_t)ncol << (4 * np);
                ++np;
            }
        }
    } else {
        for (int j = 0; j < L; ++j) {
            ord |= (uint32_t)j << (4 * j);
            colr |= (uint32_t)(j + 1) << (4 * j);
        }
        np = ncol = L;
    }
    int cnt = 0;
    uint64_t chP = 0;   // byte j: candidate set of child j
    uint32_t chv = 0;   // nibble j: its local vertex
    if (r >= 0 && 1 + ncol >= a.need) {
        uint64_t R = P;
        for (int j = np - 1; j >= 0; --j) {
            if (1 + (int)((colr >> (4 * j)) & 0xf) < a.need) break;
            const int v = (ord >> (4 * j)) & 0xf;
            const uint64_t C = R & row(v);
            R &= ~(1ull << v);
            const int pc = __popcll(C);
            if (pc == 0) {
                if (2 >= a.need) {  // {r, v} is a leaf clique of interest
                    const unsigned long long idx = atomicAdd(a.ctr + 3, 1ull);
                    if ((int64_t)idx < a.leaf_cap) {
                        a.leaf_rows[idx * 2] = __ldg(a.order + r);
                        int32_t w;
                        if constexpr (kPad) {
                            const int q = L - 1 - v;
                            w = q == 0 ? V[0] : q == 1 ? V[1] : q == 2 ? V[2] : V[3];
                        } else {
                            w = __ldg(a.ocol + vb + (L - 1 - v));
                        }
                        a.leaf_rows[idx * 2 + 1] = __ldg(a.order + w);
                    }
                }
            } else if (2 + pc >= a.need) {
                chP |= C << (8 * cnt);
                chv |= (uint32_t)v << (4 * cnt);
                ++cnt;
            }
        }
    }
    // materialise surviving roots: warp-aggregated slots for the three arrays
    const bool surv = cnt > 0;
    if (__any_sync(0xffffffffu, surv)) {
        unsigned ts, tl, tc;
        const unsigned os = warp_excl(surv ? 1u : 0u, ts);
        const unsigned ol = warp_excl(surv ? (unsigned)L : 0u, tl);
        const unsigned oc = warp_excl((unsigned)cnt, tc);
        unsigned long long bs = 0, bl = 0, bc = 0;
        if ((threadIdx.x & 31) == 0) {
            bs = atomicAdd(a.ctr + 0, (unsigned long long)ts);
            bl = atomicAdd(a.ctr + 1, (unsigned long long)tl);
            bc = atomicAdd(a.ctr + 2, (unsigned long long)tc);
        }
        bs = __shfl_sync(0xffffffffu, bs, 0) + os;
        bl = __shfl_sync(0xffffffffu, bl, 0) + ol;
        bc = __shfl_sync(0xffffffffu, bc, 0) + oc;
        if (surv) {
            if constexpr (kPad) vb = __ldg(a.orp + r);
            RootInfo ri;
            ri.r = r;
            ri.L = L;
            ri.vbase = vb;
            ri.abase = (int64_t)bl;
            a.roots[bs] = ri;
            for (int i = 0; i < L; ++i) a.adj[bl + i] = row(i);
            for (int j = 0; j < cnt; ++j) {
                a.cP[bc + j] = (chP >> (8 * j)) & 0xffull;
                a.cslot[bc + j] = (int32_t)bs;
                a.cparent[bc + j] = -1;
                a.cvloc[bc + j] = (int32_t)((chv >> (4 * j)) & 0xf);
            }
        }
    }
}

// Thread per root: roots with |N+(r)| <= 8 run root_thread on their own lane;
// longer ones (<= 64) are queued in shared memory and taken by whole warps
// (root_step<32, 2>) once the block's threads are done.
constexpr int kThreadRootMax = 8;
__global__ void __launch_bounds__(kRootWarps * 32, 4) root_expand_w1(const RootArgs a) {
    __shared__ RootSmem<64> sm_all[kRootWarps];
    __shared__ int32_t queue[kRootWarps * 32];
    __shared__ int qn;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    RootSmem<64> &sm = sm_all[wid];
    if (threadIdx.x == 0) qn = 0;
    __syncthreads();
    unsigned long long bytes = 0;  // algorithmic bytes read
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < a.count; base += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = base + threadIdx.x;
        int32_t r = i < a.count ? __ldg(a.list + i * a.stride) : -1;
        int64_t vb = 0, ve = 0;
        if (r >= 0) row_bounds(a.orp, r, vb, ve);
        const int L = (int)(ve - vb);
        if (r >= 0 && L > kThreadRootMax) {
            queue[atomicAdd(&qn, 1)] = r;
            r = -1;
        }
        if (__all_sync(0xffffffffu, r < 0 || L <= 4))
            root_thread<4>(a, r, vb, L, bytes);
        else
            root_thread<kThreadRootMax>(a, r, vb, L, bytes);
        __syncthreads();
        const int nq = qn;
        for (int q = wid; q < nq; q += kRootWarps) {
            unsigned long long wb = 0;
            root_step<32, 2>(a, queue[q], sm, wb);
            if (lane == 0) bytes += wb;
        }
        __syncthreads();
        if (threadIdx.x == 0) qn = 0;
        __syncthreads();
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) bytes += __shfl_xor_sync(0xffffffffu, bytes, o);
    if (lane == 0 && bytes) atomicAdd(a.ctr + 4, bytes);
}

// Every root of the launch has L <= 4 (the host knows the largest out-degree
// of the orientation: sparse graphs such as BA m = 4 have degeneracy 4): only
// the register-resident thread path, no queue, no barriers, and a register
// budget cut for more resident roots (ROOT_SPARSE_BLOCKS blocks per SM).
#ifndef ROOT_L4_PREFETCH
#define ROOT_L4_PREFETCH 1  // measured: 0 / 1 = 50.3 / 49.8 us on ba1m
#endif
#ifndef ROOT_SPARSE_BLOCKS
#define ROOT_SPARSE_BLOCKS 4  // measured: 4 / 5 / 6 blocks per SM = 52 / 69 / 93 us on ba1m (5, 6 spill)
#endif
__global__ void __launch_bounds__(kRootWarps * 32, ROOT_SPARSE_BLOCKS) root_expand_l4(const RootArgs a) {
    unsigned long long bytes = 0;  // algorithmic bytes read
#if ROOT_L4_PREFETCH
    // the next root id is loaded one iteration ahead (one latency off the
    // chain); with ROOT_L4_PREFETCH 2 its row bounds too
    const int64_t step = (int64_t)gridDim.x * blockDim.x;
    int64_t in = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int32_t rn = in < a.count ? __ldg(a.list + in * a.stride) : -1;
#if ROOT_L4_PREFETCH == 2
    int64_t vbn = 0, ven = 0;
    if (rn >= 0) row_bounds(a.orp, rn, vbn, ven);
#endif
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < a.count; base += step) {
        const int32_t r = rn;
        in += step;
        rn = in < a.count ? __ldg(a.list + in * a.stride) : -1;
#if ROOT_L4_PREFETCH == 2
        {
            root_thread<4, true>(a, r, vbn, (int)(ven - vbn), bytes);
            vbn = ven = 0;
            if (rn >= 0) row_bounds(a.orp, rn, vbn, ven);
            continue;
        }
#endif
#else
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < a.count; base += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = base + threadIdx.x;
        const int32_t r = i < a.count ? __ldg(a.list + i * a.stride) : -1;
#endif
        if (a.ocol4) {
            root_thread<4, true, true>(a, r, 0, 0, bytes);
            continue;
        }
        int64_t vb = 0, ve = 0;
        if (r >= 0) row_bounds(a.orp, r, vb, ve);
        root_thread<4, true>(a, r, vb, (int)(ve - vb), bytes);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) bytes += __shfl_xor_sync(0xffffffffu, bytes, o);
    if ((threadIdx.x & 31) == 0 && bytes) atomicAdd(a.ctr + 4, bytes);
}

}  // namespace

void launch_root_expand_w1(const RootArgs &a, int max_len, cudaStream_t s) {
    if (a.count <= 0) return;
#if !ROOT_NO_SPARSE
    if (max_len <= 4) {
        root_expand_l4<<<grid_for(a.count, kRootWarps * 32, 8), kRootWarps * 32, 0, s>>>(a);
        MCE_LAUNCH_CHECK();
        return;
    }
#endif
    root_expand_w1<<<grid_for(a.count, kRootWarps * 32, 8), kRootWarps * 32, 0, s>>>(a);
    MCE_LAUNCH_CHECK();
}

}  // namespace mce
