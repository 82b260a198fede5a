// Expansion kernels: every k-clique candidate (C, P) of a level is expanded
// into its (k+1)-clique candidates (PAPER.md IV-D, Algorithm 2).
//
// Layout (B200 design, not the paper's clique list): the candidates of one
// root r live in the root-local space V = N+(r) (the out-neighbours of r in
// the degeneracy orientation, so |V| <= degeneracy); a candidate set P is a
// W-word bitset over V and the root's induced adjacency is a bit matrix A
// (|V| rows x W words) built once per root with warp-cooperative sorted-list
// membership tests compacted by __ballot_sync (launch_build_adj).  Every
// deeper intersection "P after v, restricted to N(v)" (Algorithm 2 lines 4-5)
// is then one AND of W words instead of a binary search per pair.
//
// Pruning (PAPER.md II-B-3, line 63) against the running lower bound `need`:
//   bound 0: |C| + |P|                 (Algorithm 2 line 8)
//   bound 1: |C| + colours(P), greedy sequential colouring of G[P]
//            ("a tighter upper bound using ... vertex coloring"), branching
//            from the highest colour down (Tomita-Seki MCQ order), so a
//            branch is cut as soon as |C| + colour(v) < need.
// A child with an empty candidate set is a clique that cannot grow inside
// its branch: when its size reaches `need` it is recorded (leaf).
// Children go to the next level through the count pass -> scan -> write pass
// (Algorithm 2 lines 29-35: COUNTCLIQUES, CUBSCAN, OUTPUTNEWCLIQUES).
#include <cstdlib>

#include "expand.cuh"

namespace mce {

namespace {

// W == 1: one warp per root, lane i builds row i (and i+32) of the 64x64 matrix
__global__ void build_adj_w1(const RootInfo *__restrict__ roots, int64_t nroots, const int64_t *__restrict__ orp,
                             const int32_t *__restrict__ ocol, uint64_t *__restrict__ adj) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t j = warp; j < nroots; j += nwarps) {
        const RootInfo ri = roots[j];
        const int32_t *V = ocol + ri.vbase;
        for (int32_t i = lane; i < ri.L; i += 32) {
            const int32_t a = __ldg(V + i);
            uint64_t row = 0;
            // V and every out-row are sorted by CSR id, which need not follow
            // the orientation (rank) order, so both directions are checked for
            // every c: V[c] in N+(a) by one merge pass over the two sorted lists,
            // a in N+(V[c]) by binary search
            int64_t p = __ldg(orp + a), pe = __ldg(orp + a + 1);
            for (int32_t c = 0; c < ri.L && p < pe; ++c) {
                const int32_t b = __ldg(V + c);
                while (p < pe && __ldg(ocol + p) < b) ++p;
                if (p < pe && __ldg(ocol + p) == b) row |= 1ull << c;
            }
            for (int32_t c = 0; c < ri.L; ++c) {
                const int32_t b = __ldg(V + c);
                if (c != i && contains_sorted(ocol, __ldg(orp + b), __ldg(orp + b + 1), a)) row |= 1ull << c;
            }
            // local index = L-1-position (reverse degeneracy order, see expand.cuh)
            adj[ri.abase + (ri.L - 1 - i)] = __brevll(row) >> (64 - ri.L);
        }
    }
}

// W >= 2: one block per root, warp per row.  Row i of the root-local
// adjacency is N+(V[i]) ∩ V: the warp reads N+(V[i]) 32 elements at a time
// (coalesced) and every lane looks its element up in V (CSR ids order V but
// need not follow the orientation, so all of V): a hit at c sets bits (i, c)
// and (c, i).  The row stops at the first chunk beyond V[L-1].
//   Lookup: when V's id span [V[0], V[L-1]] is at most kSpanBits, V is a bit
// map over the span in shared memory with a rank per 32-bit word (position =
// rank + popc of the lower bits): two shared loads instead of a log2(L)-step
// binary search (the R-MAT hub core is a contiguous suffix of CSR-id space, so
// the spans are short); otherwise binary search in the staged V.  Bits go to
// a shared-memory bit matrix when it fits (SMEM), else straight to the
// (zeroed) global matrix.
#ifndef ADJ_CHUNKS
#define ADJ_CHUNKS 4
#endif
#ifndef ADJ_VEC
#define ADJ_VEC 1  // bit-map rows scanned with 16-byte loads (0: 32-bit loads, ADJ_CHUNKS per trip)
#endif
constexpr int kAdjChunks = ADJ_CHUNKS;
constexpr int kSpanBits = 1 << 18;
constexpr int kSpanWords = kSpanBits / 32;
template <bool SMEM>
__global__ void build_adj_block(const RootInfo *__restrict__ roots, int64_t nroots, int W,
                                const int64_t *__restrict__ orp, const int32_t *__restrict__ ocol,
                                uint64_t *__restrict__ adj, int Lmax, int use_map, unsigned long long *bytes) {
    extern __shared__ int32_t dsm[];
    // algorithmic bytes: V and the row bounds of its members
    // (4 + 16 per member), every out-row id the scan must read (4 each; a row
    // stops at the first chunk beyond V's largest id) and the matrix (8 W L)
    unsigned long long nbytes = 0;
    const int lane = threadIdx.x & 31;
    const int wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;
    int32_t *sV = dsm;
    uint32_t *sA = reinterpret_cast<uint32_t *>(dsm + ((Lmax + 3) & ~3));
    uint32_t *sMap = sA + (SMEM ? (size_t)Lmax * W * 2 : 0);
    uint16_t *sRank = reinterpret_cast<uint16_t *>(sMap + (use_map ? kSpanWords : 0));
    for (int64_t j = blockIdx.x; j < nroots; j += gridDim.x) {
        const RootInfo ri = roots[j];
        const int L = ri.L;
        uint32_t *gA = reinterpret_cast<uint32_t *>(adj + ri.abase);
        uint32_t *A = SMEM ? sA : gA;
        for (int i = threadIdx.x; i < L; i += blockDim.x) sV[i] = __ldg(ocol + ri.vbase + i);
        if (SMEM)
            for (int64_t w = threadIdx.x; w < (int64_t)L * W * 2; w += blockDim.x) sA[w] = 0u;
        __syncthreads();
        const int32_t vmin = sV[0], vmax = sV[L - 1];
        const bool map = use_map && (int64_t)vmax - vmin < kSpanBits;
        if (map) {
            const int nw = ((vmax - vmin) >> 5) + 1;
            for (int w = threadIdx.x; w < nw; w += blockDim.x) sMap[w] = 0u;
            __syncthreads();
            for (int p = threadIdx.x; p < L; p += blockDim.x) {
                const int off = sV[p] - vmin, w = off >> 5;
                atomicOr(sMap + w, 1u << (off & 31));
                // words after the previous member's word up to this one start with rank p
                const int wprev = p ? ((sV[p - 1] - vmin) >> 5) : -1;
                for (int x = wprev + 1; x <= w; ++x) sRank[x] = (uint16_t)p;
            }
            __syncthreads();
        }
        for (int i = wib; i < L; i += nwb) {
            const int32_t a = sV[i];
            const int64_t pb = __ldg(orp + a), pe = __ldg(orp + a + 1);
            if (map && ADJ_VEC) {
                // aligned 16-byte loads: a lane takes 4 consecutive ids, the warp 128
                // per trip (elements outside [pb, pe) are masked; ocol is padded by 4)
                const int li = L - 1 - i;
                int64_t q_end = pb;
                for (int64_t q0 = pb & ~3ll; q0 < pe; q0 += 128) {
                    q_end = min(pe, q0 + 128);
                    const int64_t q = q0 + 4 * lane;
                    int4 v4 = make_int4(INT32_MAX, INT32_MAX, INT32_MAX, INT32_MAX);
                    if (q < pe) v4 = __ldg(reinterpret_cast<const int4 *>(ocol + q));
                    const int32_t uu[4] = {q >= pb ? v4.x : INT32_MIN, q + 1 >= pb ? v4.y : INT32_MIN,
                                           q + 2 >= pb ? v4.z : INT32_MIN, v4.w};
                    bool past = false;
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int32_t u = q + j < pe ? uu[j] : INT32_MAX;
                        past |= u > vmax;
                        if (u >= vmin && u <= vmax) {
                            const uint32_t off = (uint32_t)(u - vmin);
                            const int w = off >> 5;
                            const uint32_t bits = sMap[w], bit = 1u << (off & 31);
                            if (bits & bit) {  // local indices L-1-position (expand.cuh)
                                const int lc = L - 1 - (sRank[w] + __popc(bits & (bit - 1u)));
                                atomicOr(A + (int64_t)li * 2 * W + (lc >> 5), 1u << (lc & 31));
                                atomicOr(A + (int64_t)lc * 2 * W + (li >> 5), 1u << (li & 31));
                            }
                        }
                    }
                    if (__any_sync(0xffffffffu, past)) break;  // sorted row: the rest is beyond V
                }
                if (lane == 0) nbytes += 20 + 4 * (unsigned long long)(q_end - pb);
                continue;
            }
            // kAdjChunks chunks of 32 ids loaded before any is looked up (the
            // row scan is bound by its load latency, one chunk per trip)
            bool stop = false;
            int64_t q_last = pb;
            for (int64_t q0 = pb; q0 < pe && !stop; q0 += 32 * kAdjChunks) {
              q_last = min(pe, q0 + 32 * kAdjChunks);
              int32_t uu[kAdjChunks];
#pragma unroll
              for (int k = 0; k < kAdjChunks; ++k) {
                  const int64_t p = q0 + 32 * k + lane;
                  uu[k] = p < pe ? __ldg(ocol + p) : INT32_MAX;
              }
#pragma unroll
              for (int k = 0; k < kAdjChunks; ++k) {
                const int32_t u = uu[k];
                if (__shfl_sync(0xffffffffu, u, 0) > vmax) {
                    stop = true;
                    break;
                }
                int c = -1;
                if (map) {
                    if (u >= vmin && u <= vmax) {
                        const int off = u - vmin, w = off >> 5;
                        const uint32_t bits = sMap[w], bit = 1u << (off & 31);
                        if (bits & bit) c = sRank[w] + __popc(bits & (bit - 1u));
                    }
                } else if (u <= vmax) {
                    int lo = 0, hi = L;
                    while (lo < hi) {
                        const int mid = (lo + hi) >> 1;
                        if (sV[mid] < u)
                            lo = mid + 1;
                        else
                            hi = mid;
                    }
                    if (lo < L && sV[lo] == u) c = lo;
                }
                if (c >= 0) {  // local indices L-1-position (expand.cuh)
                    const int li = L - 1 - i, lc = L - 1 - c;
                    atomicOr(A + (int64_t)li * 2 * W + (lc >> 5), 1u << (lc & 31));
                    atomicOr(A + (int64_t)lc * 2 * W + (li >> 5), 1u << (li & 31));
                }
              }
            }
            if (lane == 0) nbytes += 20 + 4 * (unsigned long long)(q_last - pb);
        }
        __syncthreads();
        if (SMEM) {
            for (int64_t w = threadIdx.x; w < (int64_t)L * W * 2; w += blockDim.x) gA[w] = sA[w];
        }
        if (threadIdx.x == 0) nbytes += 8ull * L * W;
        __syncthreads();
    }
    if (bytes && (threadIdx.x & 31) == 0 && nbytes) atomicAdd(bytes, nbytes);
}

__global__ void init_level1_kernel(const RootInfo *__restrict__ roots, int64_t nroots, int W, uint64_t *P,
                                   int32_t *slot, int32_t *parent, int32_t *vloc) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nroots; j += (int64_t)gridDim.x * blockDim.x) {
        const int32_t L = roots[j].L;
        for (int w = 0; w < W; ++w) {
            int32_t lo = w * 64;
            uint64_t m = L >= lo + 64 ? ~0ull : (L > lo ? ((1ull << (L - lo)) - 1) : 0ull);
            P[j * W + w] = m;
        }
        slot[j] = (int32_t)j;
        parent[j] = -1;
        vloc[j] = -1;
    }
}

// Store one leaf clique C + {v} of size k+1 (count pass).  Leaves are counted
// by the caller (aggregated per warp); a staging slot is taken only while the
// staging area has room, so a level with 10^8 maximum cliques does not
// serialise on one counter.
// Vertices (original ids) of entry e's clique C (|C| = a.k) into row[0 .. k-1]:
// the levels above the root's own space come from its prefix (a re-rooted
// candidate, reroot_build_kernel: prefix[slot * k0 ..] holds its first k0
// vertices), the rest from the chain of parent links (PAPER.md IV-B read-out).
__device__ __forceinline__ void write_path(const ExpandArgs &a, int64_t e, const RootInfo &ri, int32_t *row) {
    const int32_t *V = a.ocol + ri.vbase;
    int64_t cur = e;
    const int32_t stop = a.k0 > 0 ? a.k0 : 1;
    for (int32_t lev = a.k; lev > stop; --lev) {
        row[lev - 1] = a.order[V[ri.L - 1 - a.chain[lev].vloc[cur]]];
        cur = a.chain[lev].parent[cur];
    }
    if (a.k0 > 0) {
        const int32_t *pre = a.prefix + (int64_t)a.slot[e] * a.k0;
        for (int32_t j = 0; j < a.k0; ++j) row[j] = pre[j];
    } else {
        row[0] = a.order[ri.r];
    }
}

__device__ void store_leaf(const ExpandArgs &a, int64_t e, int32_t v, const RootInfo &ri) {
    if (*(volatile unsigned long long *)a.leaf_slot >= (unsigned long long)a.leaf_cap) return;
    const unsigned long long idx = atomicAdd(a.leaf_slot, 1ull);
    if ((int64_t)idx >= a.leaf_cap) return;
    const int32_t size = a.k + 1;
    int32_t *row = a.leaf_rows + (int64_t)idx * size;
    const int32_t *V = a.ocol + ri.vbase;
    row[a.k] = a.order[V[ri.L - 1 - v]];
    write_path(a, e, ri, row);
}

// Store one clique completion C + P of size a.need (count pass): the caller
// checked that P is a clique and k + |P| == need.  G lanes of a tile hold the
// words of P (lane gl: words gl, gl + G, ...; WPL per lane); returns with the
// row written by the whole tile.
template <int G, int WPL, bool CONTIG = false>  // CONTIG: lane gl holds words gl*WPL .. (else gl + G t)
__device__ __forceinline__ void store_clique_leaf(const ExpandArgs &a, int64_t e, const uint64_t (&P)[WPL], const RootInfo &ri,
                                  unsigned gmask) {
    const int gl = (threadIdx.x & 31) & (G - 1);
    unsigned long long idx = 0;
    if (gl == 0) {
        idx = ~0ull;
        if (*(volatile unsigned long long *)a.clq_slot < (unsigned long long)a.clq_cap) {
            idx = atomicAdd(a.clq_slot, 1ull);
            if ((int64_t)idx >= a.clq_cap) idx = ~0ull;
        }
    }
    if (G > 1) idx = __shfl_sync(gmask, idx, 0, G);
    if (idx == ~0ull) return;
    int32_t *row = a.clq_rows + (int64_t)idx * a.need;
    const int32_t *V = a.ocol + ri.vbase;
    if (gl == 0) write_path(a, e, ri, row);
    int pc = 0;
#pragma unroll
    for (int t = 0; t < WPL; ++t) pc += __popcll(P[t]);
    int incl = pc;
#pragma unroll
    for (int o = 1; o < G; o <<= 1) {
        const int y = __shfl_up_sync(gmask, incl, o, G);
        if (gl >= o) incl += y;
    }
    int pos = a.k + incl - pc;
#pragma unroll
    for (int t = 0; t < WPL; ++t) {
        uint64_t q = P[t];
        while (q) {
            const int b = __ffsll((long long)q) - 1;
            q &= q - 1;
            row[pos++] = a.order[V[ri.L - 1 - ((CONTIG ? gl * WPL + t : gl + G * t) * 64 + b)]];
        }
    }
}

// highest set bit of a W-word set (-1 if empty)
template <int W>
__device__ __forceinline__ int top_bit(const uint64_t (&C)[W]) {
    int hb = -1;
#pragma unroll
    for (int w = 0; w < W; ++w)
        if (C[w]) hb = w * 64 + 63 - __clzll((long long)C[w]);
    return hb;
}

// end-of-kernel reductions of the count pass: leaves (sum) and the highest
// candidate bit of any surviving child (max) -> the children's word stride
// ... and the deepest level any descendant can reach (max of k + 1 + |P'|)
__device__ __forceinline__ void flush_counters(const ExpandArgs &a, unsigned long long nleaf, unsigned long long nclq,
                                               int hb, int ub) {
    nleaf = __reduce_add_sync(0xffffffffu, (unsigned)nleaf);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) nclq += __shfl_xor_sync(0xffffffffu, nclq, o);
    hb = __reduce_max_sync(0xffffffffu, hb + 1) - 1;
    ub = __reduce_max_sync(0xffffffffu, ub);
    if ((threadIdx.x & 31) == 0) {
        if (nleaf) atomicAdd(a.leaf_total, nleaf);
        if (nclq) atomicAdd(a.clq_total, nclq);
        if (hb >= 0) atomicMax(a.maxbit, hb);
        if (ub > 0) atomicMax(a.maxbit + 1, ub);
    }
}

// ---------------------------------------------------------------------------
// thread per candidate, W <= 4 words (|P| bits < 256): P, the running set R
// and the child set C live in registers; the colouring order in local memory
// ---------------------------------------------------------------------------
// one candidate entry e (thread per candidate, W <= 4 words); returns its
// number of surviving children (count pass) after writing them at `out`
// (write pass).  Leaves, highest child bit and reachable depth accumulate
// into the caller's counters.
// Pair completions (thread path, reading 13): P's complement is a
// matching (every vertex of P misses at most one other), so the cliques of
// size need below (C, P) are C + one vertex of each of the m non-adjacent
// pairs + every other vertex of P: 2^m of them.  The count pass reserves
// their staging rows and records a descriptor; materialize_pairs (a block
// per descriptor) writes the rows: combination c takes the higher vertex of
// pair j when bit j of c is set.
__device__ void reserve_pair_completions(const ExpandArgs &a, int64_t e, int m) {
    if (*(volatile unsigned long long *)a.clq_slot >= (unsigned long long)a.clq_cap) return;
    const unsigned long long base = atomicAdd(a.clq_slot, 1ull << m);
    if ((int64_t)base >= a.clq_cap) return;
    const unsigned long long d = atomicAdd(a.pair_n, 1ull);
    if ((int64_t)d >= a.pair_cap) return;  // the host sees the overflow and replays with more room
    a.pair_desc[3 * d] = e;
    a.pair_desc[3 * d + 1] = (int64_t)base;
    a.pair_desc[3 * d + 2] = m;
}

constexpr int kMatThreads = 256;
__global__ void __launch_bounds__(kMatThreads) materialize_pairs_kernel(const ExpandArgs a, int64_t n) {
    __shared__ int32_t tmpl[4096];  // C + unpaired vertices (need - m <= 4096 checked by the host)
    __shared__ int32_t plo[40], phi[40];
    __shared__ int s_np2, s_len;
    for (int64_t d = blockIdx.x; d < n; d += gridDim.x) {
        const int64_t e = a.pair_desc[3 * d];
        const int64_t base = a.pair_desc[3 * d + 1];
        const int m = (int)a.pair_desc[3 * d + 2];
        if (threadIdx.x == 0) {
            const RootInfo ri = a.roots[a.slot[e]];
            const int32_t *V = a.ocol + ri.vbase;
            const uint64_t *A = a.adj + ri.abase;
            write_path(a, e, ri, tmpl);
            int pos = a.k, np2 = 0;
            for (int w = 0; w < a.Wp; ++w) {
                uint64_t q = a.P[e * a.Ps + w];
                while (q) {
                    const int b = __ffsll((long long)q) - 1;
                    q &= q - 1;
                    const int v = w * 64 + b;
                    const uint64_t *row = A + (int64_t)v * a.Wa;
                    int u = -1;
                    for (int x = 0; x < a.Wp; ++x) {
                        uint64_t nb = a.P[e * a.Ps + x] & ~row[x];
                        if (x == w) nb &= ~(1ull << b);
                        if (nb) u = x * 64 + __ffsll((long long)nb) - 1;
                    }
                    if (u < 0) {
                        tmpl[pos++] = a.order[V[ri.L - 1 - v]];
                    } else if (v < u && np2 < 40) {
                        plo[np2] = a.order[V[ri.L - 1 - v]];
                        phi[np2] = a.order[V[ri.L - 1 - u]];
                        ++np2;
                    }
                }
            }
            s_np2 = np2;
            s_len = pos;
        }
        __syncthreads();
        const int np2 = s_np2, len = s_len;
        const int64_t last = min((int64_t)(base + (1ll << m)), (int64_t)a.clq_cap);
        for (int64_t r = base + threadIdx.x; r < last; r += blockDim.x) {
            const unsigned long long c = (unsigned long long)(r - base);
            int32_t *row = a.clq_rows + r * a.need;
            for (int i = 0; i < len; ++i) row[i] = tmpl[i];
            for (int j = 0; j < np2; ++j) row[len + j] = ((c >> j) & 1ull) ? phi[j] : plo[j];
        }
        __syncthreads();
    }
}

// warp exclusive prefix sum of x over all 32 lanes (total in `total`)
__device__ __forceinline__ unsigned long long warp_excl_u64(unsigned long long x, unsigned long long &total) {
    const int lane = threadIdx.x & 31;
    unsigned long long inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    total = __shfl_sync(0xffffffffu, inc, 31);
    return inc - x;
}

// one candidate entry e (thread per candidate, W <= 4 words); returns its
// number of surviving children (count pass) after writing them at `out`
// (write pass).  Leaves, highest child bit and reachable depth accumulate
// into the caller's counters.  FUSED (count pass, called by all 32 lanes of
// the warp; `active` = lane has an entry): the children are also written, at
// slots reserved for the whole warp with one atomicAdd, by replaying the
// cheap branching loop after the colouring (which the separate write pass
// would recompute).
// adjacency row word: read-only global (LDG) or a copy in shared memory (SROWS)
template <bool SROWS>
__device__ __forceinline__ uint64_t ldrow(const uint64_t *p) {
    if constexpr (SROWS) {  // an explicit shared-space load (a generic load costs the address-window check)
        uint64_t v;
        asm("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"((unsigned)__cvta_generic_to_shared(p)));
        return v;
    } else {
        return __ldg(p);
    }
}

// SROWS: the root's rows 0 .. 64 W - 1 (first W words each) are staged at
// srows with stride W (expand_small, every candidate under one root)
constexpr int kUniCompute = -3;  // expand_entry's universal-vertex hint: compute it
constexpr int kUniAll = -2;      // P is a clique
constexpr int kUniNone = -1;     // colour as usual
#ifndef UNIVERSAL_RULE
#define UNIVERSAL_RULE 1  // 0: every candidate coloured and branched as in round 1
#endif
#ifndef THREAD_COLOUR_FLAT
#define THREAD_COLOUR_FLAT 0  // 1: one branch-free loop per class; measured slower (rmat22 chain: 624 vs 348 cycles per coloured vertex)
#endif
template <int W, bool WRITE, bool SROWS = false>
__device__ __forceinline__ int32_t expand_entry(const ExpandArgs &a, int64_t e, int64_t out, unsigned &nleaf,
                                                unsigned long long &nclq, int &hb, int &ub, bool active = true,
                                                bool fused = false, const uint64_t *srows = nullptr,
                                                int uhint = kUniCompute) {
    uint64_t P[W];
#pragma unroll
    for (int w = 0; w < W; ++w) P[w] = active ? a.P[e * a.Ps + w] : 0ull;
    RootInfo ri{};
    if (active) ri = a.roots[a.slot[e]];
    const uint64_t *A = SROWS ? srows : a.adj + ri.abase;
    const int Wa = SROWS ? W : a.Wa;
    uint8_t ord[64 * W];
    uint8_t colr[64 * W];  // colour - 1 (a full 4-word set has 256 colours)
    int np = 0;
    int ncol = 0;
    int maxcls = 0, cls_start = 0;  // largest colour class (a matching complement has classes of at most 2)
    const bool prof = a.dbg && active && e == a.begin;
    long long c0 = prof ? clock64() : 0;
    // Universal vertices (reading 19): u in P adjacent to every other
    // vertex of P is in every maximal clique below (C, P), so (C + u, P - u) is
    // the ONLY child needed -- it holds every clique of (C, P), each once -- and
    // no colouring is needed for it (its bound k + |P| is the trivial one).
    // When every vertex of P is universal, P is a clique: its colouring is one
    // class per vertex, written directly (the clique completion then applies).
    int uni = -1;       // the lowest universal vertex, if P has a non-universal one too
    bool all_uni = false;
    if (uhint != kUniCompute && active) {  // decided cooperatively by expand_small (same rule)
        uni = uhint >= 0 ? uhint : -1;
        all_uni = uhint == kUniAll;
        if (all_uni || uni >= 0) {
            int npc = 0;
#pragma unroll
            for (int w = 0; w < W; ++w) npc += __popcll(P[w]);
            if (all_uni) {
#pragma unroll
                for (int w = 0; w < W; ++w) {
                    uint64_t q = P[w];
                    while (q) {
                        const int b = __ffsll((long long)q) - 1;
                        q &= q - 1;
                        ord[np] = (uint8_t)(w * 64 + b);
                        colr[np] = (uint8_t)np;
                        ++np;
                    }
                }
                ncol = np;
                maxcls = 1;
                cls_start = np;
            } else {
                ord[0] = (uint8_t)uni;
                colr[0] = (uint8_t)(npc - 1);
                np = 1;
                ncol = npc;
                maxcls = 3;
                cls_start = np;
            }
        }
    } else if (UNIVERSAL_RULE && a.universal && a.shortcut && a.bound == 1 && active) {
        int npc = 0, nuni = 0, maxmiss = 0;
#pragma unroll
        for (int w = 0; w < W; ++w) npc += __popcll(P[w]);
        // (only near-cliques -- |P| at most twice what is still needed -- are
        // scanned: elsewhere universal vertices are rare and the scan is waste)
        if (npc >= 2 && npc <= 2 * (a.need - a.k)) {
#pragma unroll
            for (int w = 0; w < W; ++w) {
                uint64_t q = P[w];
                while (q) {
                    const int b = __ffsll((long long)q) - 1;
                    q &= q - 1;
                    const int v = w * 64 + b;
                    const uint64_t *row = A + (int64_t)v * Wa;
                    int miss = 0;
#pragma unroll
                    for (int x = 0; x < W; ++x)
                        miss += __popcll(P[x] & ~ldrow<SROWS>(row + x) & ~(x == w ? 1ull << b : 0ull));
                    maxmiss = max(maxmiss, miss);
                    if (!miss) {
                        ++nuni;
                        if (uni < 0) uni = v;
                    }
                }
            }
            all_uni = nuni == npc;
            // P's complement a matching: the colouring path's pair completion
            // (reading 13) takes every clique at once -- keep that path
            if (!all_uni && maxmiss <= 1) uni = -1;
            if (all_uni) {  // P is a clique: one colour class per vertex, ascending
#pragma unroll
                for (int w = 0; w < W; ++w) {
                    uint64_t q = P[w];
                    while (q) {
                        const int b = __ffsll((long long)q) - 1;
                        q &= q - 1;
                        ord[np] = (uint8_t)(w * 64 + b);
                        colr[np] = (uint8_t)np;
                        ++np;
                    }
                }
                ncol = np;
                maxcls = 1;
                cls_start = np;
                uni = -1;
            } else if (uni >= 0) {  // the single child on u; its bound k + 1 + (|P| - 1)
                ord[0] = (uint8_t)uni;
                colr[0] = (uint8_t)(npc - 1);
                np = 1;
                ncol = npc;
                maxcls = 3;  // (no pair completion at this level)
                cls_start = np;
            }
        }
    }
    if (a.bound == 1 && !all_uni && uni < 0) {
        uint64_t U[W];
#pragma unroll
        for (int w = 0; w < W; ++w) U[w] = P[w];
        while (true) {
            bool any = false;
#pragma unroll
            for (int w = 0; w < W; ++w) any |= U[w] != 0;
            if (!any) break;
            maxcls = max(maxcls, np - cls_start);
            cls_start = np;
            ++ncol;
            uint64_t Q[W];
#pragma unroll
            for (int w = 0; w < W; ++w) Q[w] = U[w];
#if THREAD_COLOUR_FLAT
            // one loop per class, the lowest candidate found branch-free over the
            // W words: near-clique sets (R-MAT hub chains) have mostly singleton
            // classes, where the per-word loops cost more than the colouring
            while (true) {
                int v = -1;
#pragma unroll
                for (int w = W - 1; w >= 0; --w)
                    if (Q[w]) v = w * 64 + __ffsll((long long)Q[w]) - 1;
                if (v < 0) break;
                const uint64_t *row = A + (int64_t)v * Wa;
                const uint64_t bit = 1ull << (v & 63);
#pragma unroll
                for (int x = 0; x < W; ++x) {
                    const uint64_t sel = x == (v >> 6) ? bit : 0ull;
                    Q[x] &= ~(ldrow<SROWS>(row + x) | sel);
                    U[x] &= ~sel;
                }
                ord[np] = (uint8_t)v;
                colr[np] = (uint8_t)(ncol - 1);
                ++np;
            }
#else
#pragma unroll
            for (int w = 0; w < W; ++w) {
                while (Q[w]) {
                    const int b = __ffsll((long long)Q[w]) - 1;
                    const int v = w * 64 + b;
                    const uint64_t *row = A + (int64_t)v * Wa;
#pragma unroll
                    for (int x = 0; x < W; ++x) Q[x] &= ~ldrow<SROWS>(row + x);
                    Q[w] &= ~(1ull << b);
                    U[w] &= ~(1ull << b);
                    ord[np] = (uint8_t)v;
                    colr[np] = (uint8_t)(ncol - 1);
                    ++np;
                }
            }
#endif
        }
    } else if (a.bound != 1) {
#pragma unroll
        for (int w = 0; w < W; ++w) {
            uint64_t q = P[w];
            while (q) {
                const int b = __ffsll((long long)q) - 1;
                q &= q - 1;
                ord[np] = (uint8_t)(w * 64 + b);
                colr[np] = (uint8_t)np;
                ++np;
            }
        }
        ncol = np;
    }
    if (prof) {
        const long long c1 = clock64();
        a.dbg[0] += c1 - c0;
        c0 = c1;
    }
    // P is a clique iff every colour class is a single vertex (reading 10)
    bool done = false;
    if (a.shortcut && a.bound == 1 && np >= 2 && ncol == np && a.k + np == a.need) {
        if (!WRITE) {
            ++nclq;
            store_clique_leaf<1, W>(a, e, P, ri, 0xffffffffu);
        }
        done = true;
        if (!fused) return 0;
    }
    // P's complement a matching with |C| + #colours == need: 2^m completions
    // (the greedy colouring then makes every colour class a pair or a single
    // vertex, so #colours = |P| - m; a class of three or more rules it out
    // without the pairwise test)
    maxcls = max(maxcls, np - cls_start);
    if (!done && a.shortcut && a.bound == 1 && ncol < np && np - ncol <= 40 && a.k + ncol == a.need &&
        a.need <= 4096 && maxcls <= 2) {
        bool matching = true;
        for (int i = 0; i < np && matching; ++i) {
            const int v = ord[i];
            const uint64_t *row = A + (int64_t)v * Wa;
            int miss = 0;
#pragma unroll
            for (int x = 0; x < W; ++x) {
                uint64_t nb = P[x] & ~ldrow<SROWS>(row + x);
                if (x == (v >> 6)) nb &= ~(1ull << (v & 63));
                miss += __popcll(nb);
            }
            matching = miss <= 1;
        }
        if (matching) {
            if (!WRITE) {
                nclq += 1ull << (np - ncol);
                reserve_pair_completions(a, e, np - ncol);
            }
            done = true;
            if (!fused) return 0;
        }
    }
    if (prof) {
        const long long c1 = clock64();
        a.dbg[1] += c1 - c0;
        c0 = c1;
    }
    // the branching loop (Algorithm 2 lines 3-9 with the colouring order):
    // MODE 0 count (+ leaves), 1 write at `at` with word stride `ws`
    auto branch = [&](int mode, int64_t at, int ws) -> int32_t {
        int32_t cnt = 0;
        if (done || a.k + ncol < a.need) return 0;
        uint64_t R[W];
#pragma unroll
        for (int w = 0; w < W; ++w) R[w] = P[w];
        for (int i = np - 1; i >= 0; --i) {
            if (a.k + 1 + colr[i] < a.need) break;
            const int v = ord[i];
            const uint64_t *row = A + (int64_t)v * Wa;
            uint64_t C[W];
            int pc = 0;
#pragma unroll
            for (int w = 0; w < W; ++w) {
                C[w] = R[w] & ldrow<SROWS>(row + w);
                pc += __popcll(C[w]);
            }
            R[v >> 6] &= ~(1ull << (v & 63));
            if (pc == 0) {
                if (mode == 0 && a.k + 1 >= a.need) {
                    ++nleaf;
                    store_leaf(a, e, v, ri);
                }
            } else if (a.k + 1 + pc >= a.need) {
                if (mode == 1) {
                    const int64_t c = at + cnt;
#pragma unroll
                    for (int w = 0; w < W; ++w)
                        if (w < ws) a.cP[c * ws + w] = C[w];
                    a.cslot[c] = a.slot[e];
                    a.cparent[c] = (int32_t)e;
                    a.cvloc[c] = v;
                } else {
                    hb = max(hb, top_bit<W>(C));
                    ub = max(ub, a.k + 1 + pc);
                }
                ++cnt;
            }
        }
        return cnt;
    };
    if (WRITE) return branch(1, out, a.Wc);
    const int32_t cnt = branch(0, 0, 0);
    if (prof) {
        const long long c1 = clock64();
        a.dbg[2] += c1 - c0;
        a.dbg[3] += np;
        c0 = c1;
    }
    if (fused) {
        unsigned long long total;
        const unsigned long long excl = warp_excl_u64((unsigned long long)cnt, total);
        unsigned long long base = 0;
        if ((threadIdx.x & 31) == 0 && total) base = atomicAdd(a.out_count, total);
        base = __shfl_sync(0xffffffffu, base, 0) + excl;
        if (cnt > 0 && (int64_t)(base + cnt) <= a.out_cap) branch(1, (int64_t)base, W);
    }
    return cnt;
}

template <int W, bool WRITE>
__global__ void __launch_bounds__(256) expand_thread(const ExpandArgs a) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    unsigned nleaf = 0;
    unsigned long long nclq = 0;
    int hb = -1, ub = 0;
    if (!WRITE && a.fused) {  // warp-uniform loop: the whole warp reserves its children's slots at once
        for (int64_t e0 = a.begin + (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); e0 < a.end;
             e0 += stride) {
            const int64_t e = e0 + (threadIdx.x & 31);
            const bool active = e < a.end;
            const int32_t cnt = expand_entry<W, false>(a, e, 0, nleaf, nclq, hb, ub, active, true);
            if (active) a.counts[e] = cnt;
        }
        flush_counters(a, nleaf, nclq, hb, ub);
        return;
    }
    for (int64_t e = a.begin + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < a.end; e += stride) {
        int64_t out = 0;
        if (WRITE) {
            out = a.offsets[e];
            if (a.offsets[e + 1] == out) continue;
            out -= a.out_base;
        }
        const int32_t cnt = expand_entry<W, WRITE>(a, e, out, nleaf, nclq, hb, ub);
        if (!WRITE) a.counts[e] = cnt;
    }
    if (!WRITE) flush_counters(a, nleaf, nclq, hb, ub);
}

// ---------------------------------------------------------------------------
// small-frontier fused levels (see expand.cuh)
// ---------------------------------------------------------------------------
constexpr int kSmallThreads = 512;  // (1024 capped the colouring loop at 64 registers: Q/U spilled, ~360 cycles a step)
constexpr int kSmallPer = kSmallMax / kSmallThreads;  // candidates per thread
constexpr int kSmallCoop = 16;  // levels of at most this many candidates take the block's universal-vertex scan
constexpr int kSmallRoots = 4;  // roots whose rows expand_small stages in shared memory (8 KB each)

template <bool WRITE>
__device__ __forceinline__ int32_t expand_entry_w(int W, const ExpandArgs &a, int64_t e, int64_t out,
                                                  unsigned &nleaf, unsigned long long &nclq, int &hb, int &ub,
                                                  bool active = true, bool fused = false,
                                                  const uint64_t *srows = nullptr, int uhint = kUniCompute) {
    if (srows) {
        if (W == 1) return expand_entry<1, WRITE, true>(a, e, out, nleaf, nclq, hb, ub, active, fused, srows, uhint);
        if (W == 2) return expand_entry<2, WRITE, true>(a, e, out, nleaf, nclq, hb, ub, active, fused, srows, uhint);
        return expand_entry<4, WRITE, true>(a, e, out, nleaf, nclq, hb, ub, active, fused, srows, uhint);
    }
    if (W == 1) return expand_entry<1, WRITE>(a, e, out, nleaf, nclq, hb, ub, active, fused);
    if (W == 2) return expand_entry<2, WRITE>(a, e, out, nleaf, nclq, hb, ub, active, fused);
    return expand_entry<4, WRITE>(a, e, out, nleaf, nclq, hb, ub, active, fused);
}

__global__ void __launch_bounds__(kSmallThreads, 1) expand_small(const ExpandArgs a0, uint8_t *scratch,
                                                              int64_t scratch_bytes, SmallOut *out,
                                                              LevelLink *chain) {
    __shared__ ExpandArgs A;
    __shared__ unsigned s_leaf;
    __shared__ unsigned long long s_clq, s_cnt;
    __shared__ int64_t s_end;
    __shared__ int s_hb, s_ub;
    __shared__ int64_t s_used;
    __shared__ int s_slots[kSmallRoots], s_over;
    __shared__ int s_umin, s_unum, s_umiss, s_uhint[kSmallCoop];
    __shared__ uint64_t s_rows[kSmallRoots][256 * 4];  // per root: rows 0 .. 64 W - 1, W words each (W <= 4)
    const int t = threadIdx.x;
    if (t == 0) {
        A = a0;
        s_used = 0;
        out->levels = 0;
        out->leaves = 0;
        out->cliques = 0;
        out->status = 2;
        out->k_next = a0.k;
        out->children = a0.end - a0.begin;
        out->Wc = a0.Wp;
        out->Ps = a0.Ps;
        out->P = const_cast<uint64_t *>(a0.P);
        out->slot = const_cast<int32_t *>(a0.slot);
        out->parent = const_cast<int32_t *>(a0.parent);
        out->vloc = const_cast<int32_t *>(a0.vloc);
    }
    __syncthreads();
    long long pt = clock64();
    auto phase = [&](int i) {  // thread 0: cycles since the previous mark into prof[i]
        if (t == 0) {
            const long long now = clock64();
            out->prof[i] += now - pt;
            pt = now;
        }
    };
    if (t == 0) {
        for (int i = 0; i < 10; ++i) out->prof[i] = 0;
        A.dbg = out->prof + 6;
    }
    __syncthreads();
    for (int lev = 0; lev < kSmallMaxLevels; ++lev) {
        const int64_t N = A.end - A.begin;
        const int W = A.Wp;
        // worst case of the children: every candidate bit a child
        const int64_t worst = N * 64 * W * (8 * W + 12) + 4 * 256;
        if (N > kSmallMax || W > 4 || s_used + worst > scratch_bytes) break;  // status 2: host takes level k
        if (t == 0) {
            s_leaf = 0;
            s_clq = 0;
            s_hb = -1;
            s_ub = 0;
            chain[A.k] = LevelLink{A.parent, A.vloc};
        }
        __syncthreads();
        // fused count + write, one candidate per thread: the children go to
        // worst-case arrays (every candidate bit a child) at slots reserved
        // per warp, then are compacted behind P
        if (t == 0) {
            const int64_t cap = N * 64 * W;
            uint8_t *p = scratch + s_used;
            auto take = [&](int64_t bytes) {
                uint8_t *q = p;
                p += (bytes + 255) / 256 * 256;
                return q;
            };
            A.cP = reinterpret_cast<uint64_t *>(take(cap * W * 8));
            A.cslot = reinterpret_cast<int32_t *>(take(cap * 4));
            A.cparent = reinterpret_cast<int32_t *>(take(cap * 4));
            A.cvloc = reinterpret_cast<int32_t *>(take(cap * 4));
            A.out_cap = cap;
            A.out_count = &s_cnt;
            A.fused = 1;
            s_cnt = 0;
            s_end = p - scratch;
        }
        __syncthreads();
        // candidates under at most kSmallRoots roots (the deep chains below the
        // hub roots): the roots' rows are staged in shared memory, so the
        // colouring's dependent row loads are shared-memory hits instead of
        // L2 round trips
        phase(0);
        if (t < kSmallRoots) s_slots[t] = -1;
        if (t == 0) s_over = 0;
        __syncthreads();
        int mys[kSmallPer];
#pragma unroll
        for (int r = 0; r < kSmallPer; ++r) {
            int my = -1;
            const int idx = t + r * kSmallThreads;
            if (idx < N) {
                const int32_t sl = A.slot[A.begin + idx];
                for (int j = 0; j < kSmallRoots && my < 0; ++j) {
                    const int old = atomicCAS(&s_slots[j], -1, sl);
                    if (old == -1 || old == sl) my = j;
                }
                if (my < 0) s_over = 1;
            }
            mys[r] = my;
        }
        __syncthreads();
        const bool staged = !s_over;
        if (staged) {
            for (int j = 0; j < kSmallRoots; ++j) {
                if (s_slots[j] < 0) break;
                const RootInfo ri = A.roots[s_slots[j]];
                const int nr = min(64 * W, ri.L);
                for (int q = t; q < nr * W; q += blockDim.x) {
                    const int r = q / W, x = q - r * W;
                    s_rows[j][q] = __ldg(A.adj + ri.abase + (int64_t)r * A.Wa + x);
                }
            }
        }
        __syncthreads();
        // levels of a few candidates (the deep chains): the universal-vertex scan
        // of each candidate by the whole block, one vertex per thread (a single
        // thread's scan is a chain of dependent instructions, ~200 cycles per
        // vertex); the entries then take the decision as a hint (same rule)
        const bool coop = UNIVERSAL_RULE && staged && N <= kSmallCoop && A.universal && A.shortcut && A.bound == 1;
        if (coop) {
            for (int c = 0; c < N; ++c) {
                const int64_t ec = A.begin + c;
                int cj = 0;  // the staged root of candidate c
                const int32_t slc = A.slot[ec];
                for (int j = 0; j < kSmallRoots; ++j)
                    if (s_slots[j] == slc) cj = j;
                if (t == 0) {
                    s_umin = INT32_MAX;
                    s_unum = 0;
                    s_umiss = 0;
                }
                __syncthreads();
                int npc = 0;
                uint64_t Pc[4] = {0, 0, 0, 0};
#pragma unroll
                for (int w = 0; w < 4; ++w)
                    if (w < W) {
                        Pc[w] = A.P[ec * A.Ps + w];
                        npc += __popcll(Pc[w]);
                    }
                const bool scan = npc >= 2 && npc <= 2 * (A.need - A.k);
                if (scan && t < 64 * W && ((Pc[t >> 6] >> (t & 63)) & 1ull)) {
                    const uint64_t *row = s_rows[cj] + (int64_t)t * W;
                    int miss = 0;
#pragma unroll
                    for (int x = 0; x < 4; ++x)
                        if (x < W) miss += __popcll(Pc[x] & ~row[x] & ~(x == (t >> 6) ? 1ull << (t & 63) : 0ull));
                    atomicMax(&s_umiss, miss);
                    if (!miss) {
                        atomicAdd(&s_unum, 1);
                        atomicMin(&s_umin, t);
                    }
                }
                __syncthreads();
                if (t == 0) {
                    int h = kUniNone;
                    if (scan) {
                        if (s_unum == npc)
                            h = kUniAll;
                        else if (s_unum > 0 && s_umiss > 1)
                            h = s_umin;
                    }
                    s_uhint[c] = h;
                }
                __syncthreads();
            }
        }
        phase(1);
        unsigned nleaf = 0;
        unsigned long long nclq = 0;
        int hb = -1, ub = 0;
#pragma unroll
        for (int r = 0; r < kSmallPer; ++r) {
            if (r * kSmallThreads >= N) break;  // (block-uniform)
            const int idx = t + r * kSmallThreads;
            expand_entry_w<false>(W, A, A.begin + idx, 0, nleaf, nclq, hb, ub, idx < N, true,
                                  staged ? s_rows[max(mys[r], 0)] : nullptr,  // block-uniform path
                                  coop && idx < N ? s_uhint[idx] : kUniCompute);
        }
        phase(2);  // (thread 0's own entries)
        if (nleaf) atomicAdd(&s_leaf, nleaf);
        if (nclq) atomicAdd(&s_clq, nclq);
        if (hb >= 0) atomicMax(&s_hb, hb);
        if (ub > 0) atomicMax(&s_ub, ub);
        __syncthreads();
        phase(3);  // (waiting for the block's slowest entry)
        const int64_t total = (int64_t)s_cnt;
        if (t == 0) {
            out->level_n[lev] = N;
            out->levels = lev + 1;
            out->leaves = s_leaf;
            out->cliques = s_clq;
            out->inP = const_cast<uint64_t *>(A.P);
            out->inslot = const_cast<int32_t *>(A.slot);
            out->inparent = const_cast<int32_t *>(A.parent);
            out->invloc = const_cast<int32_t *>(A.vloc);
            out->inN = N;
            out->inW = W;
            out->inPs = A.Ps;
            out->k_next = A.k + 1;
            out->children = total;
            if (s_leaf) atomicAdd(A.leaf_total, (unsigned long long)s_leaf);
            if (s_clq) atomicAdd(A.clq_total, (unsigned long long)s_clq);
        }
        if (total == 0) {
            if (t == 0) out->status = 0;
            break;
        }
        // compaction: slot / parent / vloc right behind the used part of P
        // (the new ranges end before the old ones start when total <= cap / 2)
        const int64_t cap = N * 64 * W;
        if (total <= cap / 2) {
            uint8_t *base = reinterpret_cast<uint8_t *>(A.cP);
            auto at = [&](int64_t off) { return base + (off + 255) / 256 * 256; };
            int32_t *ns = reinterpret_cast<int32_t *>(at(total * W * 8));
            int32_t *np_ = reinterpret_cast<int32_t *>(at(reinterpret_cast<uint8_t *>(ns) - base + total * 4));
            int32_t *nv = reinterpret_cast<int32_t *>(at(reinterpret_cast<uint8_t *>(np_) - base + total * 4));
            for (int64_t i = t; i < total; i += blockDim.x) ns[i] = A.cslot[i];
            __syncthreads();
            for (int64_t i = t; i < total; i += blockDim.x) np_[i] = A.cparent[i];
            __syncthreads();
            for (int64_t i = t; i < total; i += blockDim.x) nv[i] = A.cvloc[i];
            __syncthreads();
            if (t == 0) {
                A.cslot = ns;
                A.cparent = np_;
                A.cvloc = nv;
                s_used = (reinterpret_cast<uint8_t *>(nv) - scratch) + (total * 4 + 255) / 256 * 256;
            }
        } else if (t == 0) {
            s_used = s_end;
        }
        if (t == 0) {
            int Wc = 1;
            while (Wc * 64 <= s_hb && Wc < W) Wc <<= 1;
            A.Wc = Wc;
        }
        __syncthreads();
        const bool stop = s_leaf > 0 || s_clq > 0 || total > kSmallMax;
        if (t == 0) {
            out->P = A.cP;
            out->slot = A.cslot;
            out->parent = A.cparent;
            out->vloc = A.cvloc;
            out->Wc = A.Wc;
            out->Ps = A.Wp;
            out->status = 1;
            // the children become the next level
            A.P = A.cP;
            A.slot = A.cslot;
            A.parent = A.cparent;
            A.vloc = A.cvloc;
            A.begin = 0;
            A.end = total;
            A.Ps = A.Wp;  // written with the parent's width
            A.Wp = A.Wc;
            A.k = A.k + 1;
        }
        __syncthreads();
        phase(4);
        if (stop) break;
    }
}

// ---------------------------------------------------------------------------
// tile of G lanes per candidate, 4 < W <= 256 words: lane j of the tile owns
// words j, j + G, ... (WPL words per lane).  Launched with G = 32 (a warp per
// candidate); G = 8 / 16 put several candidates in one warp but diverge.
// ---------------------------------------------------------------------------
template <int G, int WPL, bool WRITE>
__global__ void expand_tile(const ExpandArgs a, int max_l) {
    extern __shared__ uint16_t sm[];
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1), gbase = lane & ~(G - 1);
    const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
    const int tib = threadIdx.x / G;  // tile in block
    uint16_t *ord = sm + (int64_t)tib * 2 * max_l;
    uint16_t *colr = ord + max_l;
    const int64_t tile = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / G;
    const int64_t ntiles = ((int64_t)gridDim.x * blockDim.x) / G;
    const int W = a.Wp, Wa = a.Wa;
    unsigned nleaf = 0;
    unsigned long long nclq = 0;
    int hb = -1, ub = 0;
    for (int64_t e = a.begin + tile; e < a.end; e += ntiles) {
        int64_t out = 0;
        if (WRITE) {
            out = a.offsets[e];
            if (a.offsets[e + 1] == out) continue;
            out -= a.out_base;
        }
        uint64_t P[WPL];
#pragma unroll
        for (int t = 0; t < WPL; ++t) {
            const int j = gl + G * t;
            P[t] = j < W ? a.P[e * a.Ps + j] : 0ull;
        }
        const RootInfo ri = a.roots[a.slot[e]];
        const uint64_t *A = a.adj + ri.abase;
        int np = 0, ncol = 0;
        if (a.bound == 1) {
            uint64_t U[WPL];
#pragma unroll
            for (int t = 0; t < WPL; ++t) U[t] = P[t];
            while (true) {
                bool any = false;
#pragma unroll
                for (int t = 0; t < WPL; ++t) any |= U[t] != 0;
                if (!((__ballot_sync(gmask, any) & gmask))) break;
                ++ncol;
                uint64_t Q[WPL];
#pragma unroll
                for (int t = 0; t < WPL; ++t) Q[t] = U[t];
                while (true) {
                    int v = -1;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) {
                        if (v < 0) {
                            const unsigned m = (__ballot_sync(gmask, Q[t] != 0) & gmask) >> gbase;
                            if (m) {
                                const int src = __ffs(m) - 1;
                                const int bit = __shfl_sync(gmask, __ffsll((long long)Q[t]) - 1, src, G);
                                v = (src + G * t) * 64 + bit;
                            }
                        }
                    }
                    if (v < 0) break;
                    const uint64_t *row = A + (int64_t)v * Wa;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) {
                        const int j = gl + G * t;
                        if (j < W) Q[t] &= ~__ldg(row + j);
                    }
                    const int jv = v >> 6;
                    if ((jv & (G - 1)) == gl) {
#pragma unroll
                        for (int t = 0; t < WPL; ++t)
                            if (t == jv / G) {
                                Q[t] &= ~(1ull << (v & 63));
                                U[t] &= ~(1ull << (v & 63));
                            }
                    }
                    if (gl == 0) {
                        ord[np] = (uint16_t)v;
                        colr[np] = (uint16_t)ncol;
                    }
                    ++np;
                }
            }
        } else {
            // ascending bit order; colr[i] = i + 1
            int base = 0;
#pragma unroll
            for (int t = 0; t < WPL; ++t) {
                const int pc = __popcll(P[t]);
                int incl = pc;
#pragma unroll
                for (int o = 1; o < G; o <<= 1) {
                    int y = __shfl_up_sync(gmask, incl, o, G);
                    if (gl >= o) incl += y;
                }
                int pos = base + incl - pc;
                uint64_t q = P[t];
                while (q) {
                    const int b = __ffsll((long long)q) - 1;
                    q &= q - 1;
                    ord[pos] = (uint16_t)((gl + G * t) * 64 + b);
                    colr[pos] = (uint16_t)(pos + 1);
                    ++pos;
                }
                base += __shfl_sync(gmask, incl, G - 1, G);
            }
            np = base;
            ncol = np;
        }
        __syncwarp(gmask);
        if (a.shortcut && a.bound == 1 && np >= 2 && ncol == np && a.k + np == a.need) {
            if (!WRITE) {
                if (gl == 0) ++nclq;
                store_clique_leaf<G, WPL>(a, e, P, ri, gmask);
                if (gl == 0) a.counts[e] = 0;
            }
            __syncwarp(gmask);
            continue;
        }
        int32_t cnt = 0;
        if (a.k + ncol >= a.need) {
            uint64_t R[WPL];
#pragma unroll
            for (int t = 0; t < WPL; ++t) R[t] = P[t];
            for (int i = np - 1; i >= 0; --i) {
                if (a.k + colr[i] < a.need) break;
                const int v = ord[i];
                const uint64_t *row = A + (int64_t)v * Wa;
                uint64_t C[WPL];
                int pc = 0;
#pragma unroll
                for (int t = 0; t < WPL; ++t) {
                    const int j = gl + G * t;
                    C[t] = j < W ? (R[t] & __ldg(row + j)) : 0ull;
                    pc += __popcll(C[t]);
                }
#pragma unroll
                for (int o = G / 2; o > 0; o >>= 1) pc += __shfl_xor_sync(gmask, pc, o, G);
                const int jv = v >> 6;
                if ((jv & (G - 1)) == gl) {
#pragma unroll
                    for (int t = 0; t < WPL; ++t)
                        if (t == jv / G) R[t] &= ~(1ull << (v & 63));
                }
                if (pc == 0) {
                    if (!WRITE && a.k + 1 >= a.need && gl == 0) {
                        ++nleaf;
                        store_leaf(a, e, v, ri);
                    }
                } else if (a.k + 1 + pc >= a.need) {
                    if (WRITE) {
                        const int64_t c = out + cnt;
#pragma unroll
                        for (int t = 0; t < WPL; ++t) {
                            const int j = gl + G * t;
                            if (j < a.Wc) a.cP[c * a.Wc + j] = C[t];
                        }
                        if (gl == 0) {
                            a.cslot[c] = a.slot[e];
                            a.cparent[c] = (int32_t)e;
                            a.cvloc[c] = v;
                        }
                    } else {
#pragma unroll
                        for (int t = 0; t < WPL; ++t)
                            if (C[t]) hb = max(hb, (gl + G * t) * 64 + 63 - __clzll((long long)C[t]));
                        ub = max(ub, a.k + 1 + pc);
                    }
                    ++cnt;
                }
            }
        }
        if (!WRITE && gl == 0) a.counts[e] = cnt;
        if (!WRITE && a.fused && cnt > 0) {  // fused: reserve and replay the branching, writing
            unsigned long long base = 0;
            if (gl == 0) base = atomicAdd(a.out_count, (unsigned long long)cnt);
            base = __shfl_sync(gmask, base, 0, G);
            if ((int64_t)(base + cnt) <= a.out_cap) {
                uint64_t R[WPL];
#pragma unroll
                for (int t = 0; t < WPL; ++t) R[t] = P[t];
                int32_t c2 = 0;
                for (int i = np - 1; i >= 0; --i) {
                    if (a.k + colr[i] < a.need) break;
                    const int v = ord[i];
                    const uint64_t *row = A + (int64_t)v * Wa;
                    uint64_t C[WPL];
                    int pc = 0;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) {
                        const int j = gl + G * t;
                        C[t] = j < W ? (R[t] & __ldg(row + j)) : 0ull;
                        pc += __popcll(C[t]);
                    }
#pragma unroll
                    for (int o = G / 2; o > 0; o >>= 1) pc += __shfl_xor_sync(gmask, pc, o, G);
                    const int jv = v >> 6;
                    if ((jv & (G - 1)) == gl) {
#pragma unroll
                        for (int t = 0; t < WPL; ++t)
                            if (t == jv / G) R[t] &= ~(1ull << (v & 63));
                    }
                    if (pc > 0 && a.k + 1 + pc >= a.need) {
                        const int64_t c = (int64_t)base + c2;
#pragma unroll
                        for (int t = 0; t < WPL; ++t) {
                            const int j = gl + G * t;
                            if (j < W) a.cP[c * W + j] = C[t];
                        }
                        if (gl == 0) {
                            a.cslot[c] = a.slot[e];
                            a.cparent[c] = (int32_t)e;
                            a.cvloc[c] = v;
                        }
                        ++c2;
                    }
                }
            }
        }
        __syncwarp(gmask);
    }
    if (!WRITE) flush_counters(a, nleaf, nclq, hb, ub);
}

// ---------------------------------------------------------------------------
// Levels >= 2 with the root's adjacency matrix staged in shared memory
// (expand_lock; W = G words per candidate set, G in {4, 8, 16}: at most 64 G
// rows of G words, 128 KB for G = 16).  The level is visited through `perm`,
// which groups its entries by root slot (launch_group_by_slot), so a block
// loads a root's matrix once per run of that root's candidates and every
// colouring / branching row read is a shared-memory hit.
//   A warp holds T = 32 / G candidates, one G-lane tile each (lane gl owns word
// gl), and runs them in LOCKSTEP: every loop is warp-uniform (it runs until
// the last tile is done, finished tiles predicated off) and every vote /
// shuffle takes the full mask, each tile reading its own G bits.  (Tiles that
// diverged instead cost ~45 warp instructions per colouring step, most of them
// the divergence checks of partial-mask collectives; a thread per candidate
// was 5x slower still: 32 unrelated serial chains diverge in a warp.)
// Count pass + fused child write, leaves, clique completions (reading 10) and
// pair completions (reading 13).
//   The colouring order is kept per tile in shared memory as u16 local
// indices with bit 15 marking the first vertex of each colour class (the
// colour of position i is recovered while walking the order backwards).
// ---------------------------------------------------------------------------
constexpr uint16_t kClassStart = 0x8000u;
constexpr unsigned kFull = 0xffffffffu;

template <int G>
__device__ __forceinline__ int tile_sum_full(int x) {  // sum over the lane's aligned G-lane tile, full-warp shuffles
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
    return x;
}
template <int G>
__device__ __forceinline__ int tile_sum(int x, unsigned gmask) {
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) x += __shfl_xor_sync(gmask, x, o, G);
    return x;
}

template <int G>
__global__ void __launch_bounds__(512) expand_lock(const ExpandArgs a, int64_t nchunks) {
    constexpr int T = 32 / G;                       // tiles (candidates) per warp
    constexpr unsigned TM = G == 32 ? kFull : ((1u << G) - 1u);
    extern __shared__ uint64_t sA[];                // [64 G rows][G words], then the tiles' colouring orders
    uint16_t *sOrd = reinterpret_cast<uint16_t *>(sA + 64 * G * G);
    __shared__ int64_t s_chunk;
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1), gbase = lane & ~(G - 1), tiw = lane / G;
    const unsigned gmask = TM << gbase;
    const int warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    uint16_t *ord = sOrd + (int64_t)(threadIdx.x / G) * 64 * G;
    const int32_t k = a.k, need = a.need;
    int32_t loaded = -1;
    unsigned nleaf = 0;
    unsigned long long nclq = 0;
    int hb = -1, ub = 0;
    for (;;) {
        if (threadIdx.x == 0) s_chunk = (int64_t)atomicAdd(a.chunk_ctr, 1ull);
        __syncthreads();
        const int64_t c = s_chunk;
        __syncthreads();
        if (c >= nchunks) break;
        const int64_t p1 = min(a.end, a.begin + (c + 1) * (int64_t)a.chunk);
        for (int64_t q0 = a.begin + c * (int64_t)a.chunk; q0 < p1;) {
            const int32_t slot = a.slot[a.perm[q0]];
            int64_t lo = q0 + 1, hi = p1;  // end of this slot's run (positions are grouped by slot)
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                if (a.slot[a.perm[mid]] == slot)
                    lo = mid + 1;
                else
                    hi = mid;
            }
            const int64_t q1 = lo;
            const RootInfo ri = a.roots[slot];
            if (slot != loaded) {  // stage the root's rows (only the first G words matter: P < 64 G bits)
                __syncthreads();
                const int rows = min(ri.L, 64 * G);
                const uint64_t *gA = a.adj + ri.abase;
                for (int w = threadIdx.x; w < rows * G; w += blockDim.x)
                    sA[w] = __ldg(gA + (int64_t)(w / G) * a.Wa + (w % G));
                __syncthreads();
                loaded = slot;
            }
            // warp-uniform trips: T candidates per warp per trip
            for (int64_t qb = q0 + (int64_t)warp * T; qb < q1; qb += (int64_t)nwarps * T) {
                const int64_t q = qb + tiw;
                const bool active = q < q1;
                const int64_t e = active ? a.perm[q] : 0;
                const uint64_t P = active ? a.P[e * a.Ps + gl] : 0ull;
                // ---- colouring, one vertex per tile per trip
                int np = 0, ncol = 0;
                if (a.bound == 1) {
                    uint64_t U = P, Q = 0ull;
                    uint16_t first = 0;
                    while (true) {
                        const unsigned bq = __ballot_sync(kFull, Q != 0ull), bu = __ballot_sync(kFull, U != 0ull);
                        if (!(bq | bu)) break;  // every tile coloured
                        unsigned mq = (bq >> gbase) & TM;
                        if (!mq) {  // this tile's class is closed: the next one starts from what is left
                            const unsigned mu = (bu >> gbase) & TM;
                            if (mu) {
                                Q = U;
                                mq = mu;
                                ++ncol;
                                first = kClassStart;
                            }
                        }
                        const int src = mq ? __ffs(mq) - 1 : 0;
                        const int bit = __shfl_sync(kFull, __ffsll((long long)Q) - 1, gbase + src);
                        if (mq) {
                            const int v = src * 64 + bit;
                            Q &= ~sA[v * G + gl];
                            if (gl == src) {
                                Q &= ~(1ull << bit);
                                U &= ~(1ull << bit);
                            }
                            if (gl == 0) ord[np] = (uint16_t)v | first;
                            first = 0;
                            ++np;
                        }
                    }
                } else {
                    const int pc = __popcll(P);
                    int incl = pc;
#pragma unroll
                    for (int o = 1; o < G; o <<= 1) {
                        const int y = __shfl_up_sync(kFull, incl, o);
                        if (gl >= o) incl += y;
                    }
                    int pos = incl - pc;
                    uint64_t q2 = P;
                    while (q2) {  // every vertex its own "class": colour of position i = i + 1
                        const int b = __ffsll((long long)q2) - 1;
                        q2 &= q2 - 1;
                        ord[pos++] = (uint16_t)(gl * 64 + b) | kClassStart;
                    }
                    np = __shfl_sync(kFull, incl, gbase + G - 1);
                    ncol = np;
                }
                __syncwarp();
                // ---- completions (rare: divergent, tile-mask collectives)
                bool done = !active;
                if (!done && a.shortcut && a.bound == 1 && np >= 2 && ncol == np && k + np == need) {
                    if (gl == 0) {  // P is a clique (reading 10)
                        ++nclq;
                        a.counts[e] = 0;
                    }
                    uint64_t Pa[1] = {P};
                    store_clique_leaf<G, 1>(a, e, Pa, ri, gmask);
                    done = true;
                }
                if (!done && a.shortcut && a.bound == 1 && ncol < np && np - ncol <= 40 && k + ncol == need &&
                    need <= 4096) {  // P's complement a matching (reading 13)
                    bool matching = true;
                    for (int i = 0; i < np && matching; ++i) {
                        const int v = ord[i] & 0x7fff;
                        uint64_t nb = P & ~sA[v * G + gl];
                        if (gl == (v >> 6)) nb &= ~(1ull << (v & 63));
                        matching = tile_sum<G>(__popcll(nb), gmask) <= 1;
                    }
                    if (matching) {
                        if (gl == 0) {
                            nclq += 1ull << (np - ncol);
                            reserve_pair_completions(a, e, np - ncol);
                            a.counts[e] = 0;
                        }
                        done = true;
                    }
                }
                __syncwarp();
                // ---- branching from the last position (highest colour) down, in lockstep
                int32_t cnt = 0;
                {
                    bool stop = done || k + ncol < need;
                    uint64_t R = P;
                    int col = ncol, pos = np - 1;
                    while (__ballot_sync(kFull, !stop)) {
                        if (!stop && (pos < 0 || k + col < need)) stop = true;
                        const uint16_t o = stop ? 0 : ord[pos];
                        const int v = o & 0x7fff;
                        const uint64_t C = stop ? 0ull : (R & sA[v * G + gl]);
                        const int pc = tile_sum_full<G>(__popcll(C));
                        if (!stop) {
                            if (o & kClassStart) --col;
                            --pos;
                            if (gl == (v >> 6)) R &= ~(1ull << (v & 63));
                            if (pc == 0) {
                                if (k + 1 >= need && gl == 0) {
                                    ++nleaf;
                                    store_leaf(a, e, v, ri);
                                }
                            } else if (k + 1 + pc >= need) {
                                if (C) hb = max(hb, gl * 64 + 63 - __clzll((long long)C));
                                ub = max(ub, k + 1 + pc);
                                ++cnt;
                            }
                        }
                    }
                }
                if (active && !done && gl == 0) a.counts[e] = cnt;
                if (a.fused) {  // reserve the warp's children at once, replay the branching, write them
                    int tot = cnt;  // exclusive scan over the warp's tiles (value held by every lane of a tile)
                    int excl = 0;
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        const int ct = __shfl_sync(kFull, cnt, t * G);
                        if (t < tiw) excl += ct;
                        if (t == 0) tot = ct; else tot += ct;
                    }
                    unsigned long long base = 0;
                    if (lane == 0 && tot) base = atomicAdd(a.out_count, (unsigned long long)tot);
                    base = __shfl_sync(kFull, base, 0) + (unsigned long long)excl;
                    const bool fits = (int64_t)(base - excl + tot) <= a.out_cap;
                    bool stop = done || cnt == 0 || !fits || k + ncol < need;
                    uint64_t R = P;
                    int col = ncol, pos = np - 1;
                    int64_t cpos = (int64_t)base;
                    while (__ballot_sync(kFull, !stop)) {
                        if (!stop && (pos < 0 || k + col < need)) stop = true;
                        const uint16_t o = stop ? 0 : ord[pos];
                        const int v = o & 0x7fff;
                        const uint64_t C = stop ? 0ull : (R & sA[v * G + gl]);
                        const int pc = tile_sum_full<G>(__popcll(C));
                        if (!stop) {
                            if (o & kClassStart) --col;
                            --pos;
                            if (gl == (v >> 6)) R &= ~(1ull << (v & 63));
                            if (pc > 0 && k + 1 + pc >= need) {
                                a.cP[cpos * G + gl] = C;
                                if (gl == 0) {
                                    a.cslot[cpos] = slot;
                                    a.cparent[cpos] = (int32_t)e;
                                    a.cvloc[cpos] = v;
                                }
                                ++cpos;
                            }
                        }
                    }
                }
                __syncwarp();
            }
            q0 = q1;
        }
    }
    flush_counters(a, nleaf, nclq, hb, ub);
}

// ---------------------------------------------------------------------------
// Re-rooting (see expand.cuh launch_reroot_build): a candidate whose set P is
// a few hundred bits scattered over a wide root space (R-MAT scale 26: roots
// of 2048-4096 out-neighbours, W = 64) becomes a root of its own over P, so
// its subtree runs at the width of |P| (4-16 words, the shared-memory pass)
// instead of the root's.  Exact: the new space keeps the old relative order,
// so colouring and branching are the same sequence of sets.
// ---------------------------------------------------------------------------
__global__ void reroot_sizes_kernel(const uint64_t *__restrict__ P, int Ps, int W, int64_t n, int32_t *Lp,
                                    int32_t *cls, unsigned long long *hist) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t e0 = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); e0 < n; e0 += stride) {
        const int64_t e = e0 + (threadIdx.x & 31);
        int32_t c = -1;
        if (e < n) {
            int pc = 0;
            for (int w = 0; w < W; ++w) pc += __popcll(P[e * Ps + w]);
            Lp[e] = pc;
            c = 0;
            while ((64 << c) < pc) ++c;
            cls[e] = c;
        }
        const unsigned same = __match_any_sync(0xffffffffu, c);
        if (c >= 0 && (threadIdx.x & 31) == __ffs(same) - 1) atomicAdd(hist + c, (unsigned long long)__popc(same));
    }
}

__global__ void gather_i32_kernel(const int32_t *__restrict__ src, const int32_t *__restrict__ idx, int64_t n,
                                  int32_t *dst) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = src[idx[i]];
}

constexpr int kRerootWarps = 8;
constexpr int kRerootMaxL = 1024;  // re-rooted spaces of at most 16 words
__global__ void __launch_bounds__(32 * kRerootWarps)
    reroot_build_kernel(const ExpandArgs a, const int32_t *__restrict__ list, int64_t cnt,
                        const int64_t *__restrict__ voff, int Wn, int32_t *nV, uint64_t *nA, RootInfo *nroots,
                        uint64_t *nP, int32_t *nslot, int32_t *nparent, int32_t *nvloc, int32_t *nprefix) {
    __shared__ uint16_t spos[kRerootWarps][kRerootMaxL];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    uint16_t *pos = spos[wib];
    for (int64_t i = (int64_t)blockIdx.x * kRerootWarps + wib; i < cnt; i += (int64_t)gridDim.x * kRerootWarps) {
        const int64_t e = list[i];
        const RootInfo ri = a.roots[a.slot[e]];
        const int32_t *Vo = a.ocol + ri.vbase;
        const uint64_t *Ao = a.adj + ri.abase;
        const int64_t base = voff[i];
        const int Lp = (int)(voff[i + 1] - base);
        // positions of P's bits, ascending (the new local indices 0 .. Lp-1)
        int np = 0;
        for (int w = 0; w < a.Wp; ++w) {
            const uint64_t word = a.P[e * a.Ps + w];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const uint32_t m = (uint32_t)(word >> (32 * h));
                if ((m >> lane) & 1u) pos[np + __popc(m & lanemask_lt())] = (uint16_t)(w * 64 + h * 32 + lane);
                np += __popc(m);
            }
        }
        __syncwarp();
        for (int j = lane; j < Lp; j += 32) nV[base + (Lp - 1 - j)] = Vo[ri.L - 1 - pos[j]];
        // rows: A'[j] = A[pos[j]] compressed to P's bits
        uint64_t *Arow = nA + base * Wn;
        const int wused = (Lp + 63) >> 6;  // words beyond are zero
        for (int j = 0; j < Lp; ++j) {
            const uint64_t *row = Ao + (int64_t)pos[j] * a.Wa;
            uint32_t lo = 0;
            if (lane >= wused && lane < Wn) Arow[(int64_t)j * Wn + lane] = 0ull;
            for (int t0 = 0; t0 < 64 * wused; t0 += 32) {
                const int t = t0 + lane;
                bool bit = false;
                if (t < Lp) {
                    const int u = pos[t];
                    bit = (__ldg(row + (u >> 6)) >> (u & 63)) & 1ull;
                }
                const uint32_t m = __ballot_sync(0xffffffffu, bit);
                if ((t0 & 32) == 0) {
                    lo = m;
                } else if (lane == 0) {
                    Arow[(int64_t)j * Wn + (t0 >> 6)] = ((uint64_t)m << 32) | lo;
                }
            }
        }
        if (lane < Wn) {
            const int lo = lane * 64;
            nP[i * Wn + lane] = Lp >= lo + 64 ? ~0ull : (Lp > lo ? ((1ull << (Lp - lo)) - 1) : 0ull);
        }
        if (lane == 0) {
            RootInfo nr;
            nr.r = ri.r;
            nr.L = Lp;
            nr.vbase = base;
            nr.abase = base * Wn;
            nroots[i] = nr;
            nslot[i] = (int32_t)i;
            nparent[i] = -1;
            nvloc[i] = -1;
            write_path(a, e, ri, nprefix + i * a.k);
        }
        __syncwarp();
    }
}

// ---------------------------------------------------------------------------
// Wide levels (W = G * WPL >= 32 words: roots of more than 1024 out-neighbours,
// R-MAT scale 26) with rows read from global memory (the L2; a 64-word root
// matrix is 2 MB): expand_lock's lockstep tiles with WPL contiguous words per
// lane (vector row loads), T = 32 / G candidates per warp in flight, and work
// taken dynamically in chunks (a static grid stride left most warps idle
// behind a few long candidates: 16% achieved occupancy, ncu).  The colouring
// order is kept only for the vertices the branching can visit (colour >= need
// - k), in per-tile global scratch (the L2), so shared memory does not cap the
// warps per SM.
// ---------------------------------------------------------------------------
template <int G, int WPL>
__global__ void __launch_bounds__(256) expand_wide(const ExpandArgs a, int64_t nchunks, uint16_t *__restrict__ scratch) {
    constexpr int T = 32 / G;
    constexpr int W = G * WPL;
    constexpr unsigned TM = G == 32 ? kFull : ((1u << G) - 1u);
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1), gbase = lane & ~(G - 1), tiw = lane / G;
    const unsigned gmask = TM << gbase;
    const int warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    uint16_t *ord = scratch + ((int64_t)blockIdx.x * (blockDim.x / G) + threadIdx.x / G) * (64 * W);
    const int32_t k = a.k, need = a.need, cmin = need - k;
    unsigned nleaf = 0;
    unsigned long long nclq = 0;
    int hb = -1, ub = 0;
    (void)warp;
    (void)nwarps;
    // every warp takes its own chunks of positions (no block barrier: a block's
    // warps never wait for its slowest candidate)
    for (;;) {
        unsigned long long c = 0;
        if (lane == 0) c = atomicAdd(a.chunk_ctr, 1ull);
        c = __shfl_sync(kFull, c, 0);
        if ((int64_t)c >= nchunks) break;
        const int64_t q0 = a.begin + (int64_t)c * a.chunk, q1 = min(a.end, q0 + (int64_t)a.chunk);
        for (int64_t qb = q0; qb < q1; qb += T) {
            const int64_t q = qb + tiw;
            const bool active = q < q1;
            const int64_t e = active ? (a.perm ? (int64_t)a.perm[q] : q) : 0;
            uint64_t P[WPL];
#pragma unroll
            for (int t = 0; t < WPL; ++t) P[t] = active ? a.P[e * a.Ps + gl * WPL + t] : 0ull;
            const int32_t slot = active ? a.slot[e] : 0;
            const RootInfo ri = a.roots[slot];
            const uint64_t *A = a.adj + ri.abase;
            // ---- colouring; the order is stored from colour cmin up
            int np = 0, ncol = 0, ns = 0;
            if (a.bound == 1) {
                uint64_t U[WPL], Q[WPL];
#pragma unroll
                for (int t = 0; t < WPL; ++t) {
                    U[t] = P[t];
                    Q[t] = 0ull;
                }
                uint16_t first = 0;
                while (true) {
                    bool qn = false, un = false;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) {
                        qn |= Q[t] != 0ull;
                        un |= U[t] != 0ull;
                    }
                    const unsigned bq = __ballot_sync(kFull, qn), bu = __ballot_sync(kFull, un);
                    if (!(bq | bu)) break;
                    unsigned mq = (bq >> gbase) & TM;
                    if (!mq) {
                        const unsigned mu = (bu >> gbase) & TM;
                        if (mu) {
#pragma unroll
                            for (int t = 0; t < WPL; ++t) Q[t] = U[t];
                            mq = mu;
                            ++ncol;
                            first = kClassStart;
                        }
                    }
                    const int src = mq ? __ffs(mq) - 1 : 0;
                    int lb = 0;  // this lane's lowest set bit (word-major)
#pragma unroll
                    for (int t = WPL - 1; t >= 0; --t)
                        if (Q[t]) lb = t * 64 + __ffsll((long long)Q[t]) - 1;
                    lb = __shfl_sync(kFull, lb, gbase + src);
                    if (mq) {
                        const int v = src * 64 * WPL + lb;
                        const uint64_t *row = A + (int64_t)v * a.Wa + gl * WPL;
#pragma unroll
                        for (int t = 0; t < WPL; ++t) Q[t] &= ~__ldg(row + t);
                        {  // clear v (select form: no dynamically indexed array, so no local memory)
                            const uint64_t bit = gl == src ? 1ull << (lb & 63) : 0ull;
                            const int wsel = lb >> 6;
#pragma unroll
                            for (int t = 0; t < WPL; ++t) {
                                const uint64_t m = wsel == t ? bit : 0ull;
                                Q[t] &= ~m;
                                U[t] &= ~m;
                            }
                        }
                        if (ncol >= cmin) {
                            if (gl == 0) ord[ns] = (uint16_t)v | first;
                            ++ns;
                        }
                        first = 0;
                        ++np;
                    }
                }
            } else {  // |C| + |P|: positions in ascending bit order, colour of position i = i + 1
                int pc = 0;
#pragma unroll
                for (int t = 0; t < WPL; ++t) pc += __popcll(P[t]);
                int incl = pc;
#pragma unroll
                for (int o = 1; o < G; o <<= 1) {
                    const int y = __shfl_up_sync(kFull, incl, o);
                    if (gl >= o) incl += y;
                }
                int pos = incl - pc;
#pragma unroll
                for (int t = 0; t < WPL; ++t) {
                    uint64_t q2 = P[t];
                    while (q2) {
                        const int b = __ffsll((long long)q2) - 1;
                        q2 &= q2 - 1;
                        ord[pos++] = (uint16_t)((gl * WPL + t) * 64 + b) | kClassStart;
                    }
                }
                np = __shfl_sync(kFull, incl, gbase + G - 1);
                ncol = np;
                ns = np;
            }
            __syncwarp();
            __threadfence_block();
            // ---- completions (rare: divergent, tile-mask collectives)
            bool done = !active;
            if (!done && a.shortcut && a.bound == 1 && np >= 2 && ncol == np && k + np == need) {
                if (gl == 0) {
                    ++nclq;
                    a.counts[e] = 0;
                }
                store_clique_leaf<G, WPL, true>(a, e, P, ri, gmask);
                done = true;
            }
            if (!done && a.shortcut && a.bound == 1 && ncol < np && np - ncol <= 40 && k + ncol == need &&
                need <= 4096) {  // P's complement a matching (reading 13): every vertex of P, one by one
                bool matching = true;
                uint64_t X[WPL];
#pragma unroll
                for (int t = 0; t < WPL; ++t) X[t] = P[t];
                while (matching) {
                    bool xn = false;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) xn |= X[t] != 0ull;
                    const unsigned mx = (__ballot_sync(gmask, xn) & gmask) >> gbase;
                    if (!mx) break;
                    const int src = __ffs(mx) - 1;
                    int lb = 0;
#pragma unroll
                    for (int t = WPL - 1; t >= 0; --t)
                        if (X[t]) lb = t * 64 + __ffsll((long long)X[t]) - 1;
                    lb = __shfl_sync(gmask, lb, src, G);
                    const int v = src * 64 * WPL + lb;
                    const uint64_t *row = A + (int64_t)v * a.Wa + gl * WPL;
                    int miss = 0;
                    const uint64_t bit = gl == src ? 1ull << (lb & 63) : 0ull;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) {
                        const uint64_t m = (lb >> 6) == t ? bit : 0ull;
                        const uint64_t nb = P[t] & ~__ldg(row + t) & ~m;
                        X[t] &= ~m;
                        miss += __popcll(nb);
                    }
                    matching = tile_sum<G>(miss, gmask) <= 1;
                }
                if (matching) {
                    if (gl == 0) {
                        nclq += 1ull << (np - ncol);
                        reserve_pair_completions(a, e, np - ncol);
                        a.counts[e] = 0;
                    }
                    done = true;
                }
            }
            __syncwarp();
            // ---- branching over the stored positions, highest colour first, in lockstep:
            // pass 0 counts (+ leaves), pass 1 (fused) writes the warp's reserved children
            int32_t cnt = 0;
            for (int pass = 0; pass < (a.fused ? 2 : 1); ++pass) {
                int64_t at = -1;
                if (pass == 1) {
                    int tot = 0, excl = 0;
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        const int ct = __shfl_sync(kFull, cnt, t * G);
                        if (t < tiw) excl += ct;
                        tot += ct;
                    }
                    unsigned long long wbase = 0;
                    if (lane == 0 && tot) wbase = atomicAdd(a.out_count, (unsigned long long)tot);
                    wbase = __shfl_sync(kFull, wbase, 0);
                    if (cnt > 0 && (int64_t)(wbase + tot) <= a.out_cap) at = (int64_t)(wbase + excl);
                }
                const bool write = pass == 1;
                int32_t c2 = 0;
                bool stop = done || k + ncol < need || (write && at < 0);
                uint64_t R[WPL];
#pragma unroll
                for (int t = 0; t < WPL; ++t) R[t] = P[t];
                int col = ncol, pos = ns - 1;
                while (__ballot_sync(kFull, !stop)) {
                    if (!stop && (pos < 0 || k + col < need)) stop = true;
                    const uint16_t o = stop ? 0 : ord[pos];
                    const int v = o & 0x7fff;
                    uint64_t C[WPL];
                    int pc = 0;
                    const uint64_t *row = A + (int64_t)v * a.Wa + gl * WPL;
#pragma unroll
                    for (int t = 0; t < WPL; ++t) {
                        C[t] = stop ? 0ull : (R[t] & __ldg(row + t));
                        pc += __popcll(C[t]);
                    }
                    pc = tile_sum_full<G>(pc);
                    if (!stop) {
                        if (o & kClassStart) --col;
                        --pos;
                        {
                            const uint64_t bit = gl == (v >> 6) / WPL ? 1ull << (v & 63) : 0ull;
                            const int wsel = (v >> 6) % WPL;
#pragma unroll
                            for (int t = 0; t < WPL; ++t) R[t] &= ~(wsel == t ? bit : 0ull);
                        }
                        if (pc == 0) {
                            if (!write && k + 1 >= need && gl == 0) {
                                ++nleaf;
                                store_leaf(a, e, v, ri);
                            }
                        } else if (k + 1 + pc >= need) {
                            if (write) {
                                const int64_t cp = at + c2;
#pragma unroll
                                for (int t = 0; t < WPL; ++t) a.cP[cp * W + gl * WPL + t] = C[t];
                                if (gl == 0) {
                                    a.cslot[cp] = slot;
                                    a.cparent[cp] = (int32_t)e;
                                    a.cvloc[cp] = v;
                                }
                            } else {
#pragma unroll
                                for (int t = 0; t < WPL; ++t)
                                    if (C[t]) hb = max(hb, (gl * WPL + t) * 64 + 63 - __clzll((long long)C[t]));
                                ub = max(ub, k + 1 + pc);
                            }
                            ++c2;
                        }
                    }
                }
                if (pass == 0) {
                    cnt = c2;
                    if (active && !done && gl == 0) a.counts[e] = cnt;
                }
            }
            __syncwarp();
        }
    }
    flush_counters(a, nleaf, nclq, hb, ub);
}

// counting sort of a level's entries by root slot (order inside a slot is
// arbitrary).  Few slots take millions of entries, so the atomics are
// aggregated over the lanes of a warp holding the same slot (__match_any_sync).
__global__ void slot_hist_kernel(const int32_t *__restrict__ slot, int64_t n, int32_t *hist) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i0 = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); i0 < n; i0 += stride) {
        const int64_t i = i0 + (threadIdx.x & 31);
        const int32_t sl = i < n ? slot[i] : -1;
        const unsigned same = __match_any_sync(0xffffffffu, sl);
        if (sl >= 0 && (threadIdx.x & 31) == __ffs(same) - 1) atomicAdd(hist + sl, __popc(same));
    }
}
__global__ void slot_scatter_kernel(const int32_t *__restrict__ slot, int64_t n, unsigned long long *cursor,
                                    int32_t *perm) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int lane = threadIdx.x & 31;
    for (int64_t i0 = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); i0 < n; i0 += stride) {
        const int64_t i = i0 + lane;
        const int32_t sl = i < n ? slot[i] : -1;
        const unsigned same = __match_any_sync(0xffffffffu, sl);
        const int leader = __ffs(same) - 1;
        unsigned long long base = 0;
        if (sl >= 0 && lane == leader) base = atomicAdd(cursor + sl, (unsigned long long)__popc(same));
        base = __shfl_sync(0xffffffffu, base, leader);
        if (sl >= 0) perm[base + __popc(same & lanemask_lt())] = (int32_t)i;
    }
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// hash of entry e's vertex path (original vertex ids, root first, then levels
// k .. 2): the same on every shard whatever local space (root or re-rooted
// candidate) the entry lives in
__global__ void shard_flags_kernel(const ExpandArgs a, int64_t n, int32_t k, int32_t rank, int32_t count,
                                   int32_t *flag) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
        const RootInfo ri = a.roots[a.slot[e]];
        const int32_t *V = a.ocol + ri.vbase;
        const int32_t *pre = a.k0 > 0 ? a.prefix + (int64_t)a.slot[e] * a.k0 : nullptr;
        uint64_t h = mix64((uint64_t)(uint32_t)(pre ? pre[0] : a.order[ri.r]));
        int64_t cur = e;
        for (int32_t lev = k; lev >= 2; --lev) {
            int32_t v;
            if (pre && lev <= a.k0) {
                v = pre[lev - 1];
            } else {
                v = a.order[V[ri.L - 1 - a.chain[lev].vloc[cur]]];
                cur = a.chain[lev].parent[cur];
            }
            h = mix64(h ^ (uint64_t)(uint32_t)v);
        }
        flag[e] = (int32_t)(h % (uint64_t)count) == rank;
    }
}

__global__ void gather_level_kernel(int64_t n, const int32_t *__restrict__ flag, const int64_t *__restrict__ pos,
                                    int W, int Ps, const uint64_t *__restrict__ P, const int32_t *__restrict__ slot,
                                    const int32_t *__restrict__ parent, const int32_t *__restrict__ vloc,
                                    uint64_t *oP, int32_t *oslot, int32_t *oparent, int32_t *ovloc) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
        if (!flag[e]) continue;
        const int64_t o = pos[e];
        for (int w = 0; w < W; ++w) oP[o * W + w] = P[e * Ps + w];
        oslot[o] = slot[e];
        oparent[o] = parent[e];
        ovloc[o] = vloc[e];
    }
}

__global__ void classify_roots_kernel(int64_t n, const int64_t *__restrict__ orp, int32_t min_len,
                                      int32_t shard_rank, int32_t shard_count, const uint8_t *__restrict__ keep,
                                      int64_t keep_T, int32_t *cls, unsigned long long *hist) {
    __shared__ unsigned int h[kMaxClass + 1];
    for (int i = threadIdx.x; i <= kMaxClass; i += blockDim.x) h[i] = 0;
    __syncthreads();
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t L = orp[r + 1] - orp[r];
        int32_t c = -1;
        if (L >= min_len && L > 0 && (shard_count <= 1 || r % shard_count == shard_rank) &&
            (!keep || (r >= keep_T && keep[r - keep_T]))) {
            const int64_t words = (L + 63) / 64;
            c = 0;
            while ((1ll << c) < words) ++c;
            if (c >= kMaxClass) c = kMaxClass;
            atomicAdd(&h[c], 1u);
        }
        cls[r] = c;
    }
    __syncthreads();
    for (int i = threadIdx.x; i <= kMaxClass; i += blockDim.x)
        if (h[i]) atomicAdd(hist + i, (unsigned long long)h[i]);
}

__global__ void flag_eq_kernel(int64_t n, const int32_t *__restrict__ cls, int32_t c, int32_t *flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        flag[i] = cls[i] == c;
}

__global__ void compact_idx_kernel(int64_t n, const int32_t *__restrict__ flag, const int64_t *__restrict__ pos,
                                   int32_t *out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (flag[i]) out[pos[i]] = (int32_t)i;
}

__global__ void root_lengths_kernel(const int32_t *__restrict__ list, int64_t count, int64_t stride,
                                    const int64_t *__restrict__ orp, int32_t *len) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = list[i * stride];
        len[i] = (int32_t)(orp[r + 1] - orp[r]);
    }
}

__global__ void make_roots_kernel(const int32_t *__restrict__ list, int64_t count, int64_t stride, int W,
                                  const int64_t *__restrict__ orp, const int64_t *__restrict__ row_prefix,
                                  RootInfo *roots) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = list[i * stride];
        RootInfo ri;
        ri.r = r;
        ri.vbase = orp[r];
        ri.L = (int32_t)(orp[r + 1] - ri.vbase);
        ri.abase = (row_prefix[i] - row_prefix[0]) * W;
        roots[i] = ri;
    }
}

// largest b in (a, n] with offsets[b] - offsets[a] <= cap (at least a+1 if possible)
__global__ void find_chunk_end_kernel(const int64_t *__restrict__ offsets, int64_t a, int64_t n, int64_t cap,
                                      int64_t *out) {
    const int64_t base = offsets[a];
    int64_t lo = a, hi = n;  // invariant: offsets[lo]-base <= cap
    while (lo < hi) {
        int64_t mid = (lo + hi + 1) >> 1;
        if (offsets[mid] - base <= cap)
            lo = mid;
        else
            hi = mid - 1;
    }
    out[0] = lo;
    out[1] = offsets[lo] - base;
    out[2] = base;
}

// smallest lo in [lo_min, hi) whose roots [lo, hi) fit `room` bytes (at least hi - 1)
__global__ void find_window_kernel(const int64_t *__restrict__ prefix, int64_t hi, int64_t lo_min, int64_t room,
                                   int64_t row_bytes, int64_t per_root, int64_t *out) {
    int64_t l = lo_min, h = hi - 1;
    while (l < h) {
        const int64_t mid = (l + h) >> 1;
        const int64_t bytes = (prefix[hi] - prefix[mid]) * row_bytes + (hi - mid) * per_root;
        if (bytes <= room)
            h = mid;
        else
            l = mid + 1;
    }
    out[0] = l;
    out[1] = prefix[hi] - prefix[l];
}

template <int G, int WPL>
void launch_tile(const ExpandArgs &a, bool write_pass, cudaStream_t s) {
    const int max_l = 64 * a.Wp;
    // 32 KB of colouring order per block: (threads / G) tiles x 2 x 64 W x 2 B
    const int threads = WPL >= 4 ? 32 : (WPL == 2 ? 64 : 128);
    const size_t smem = (size_t)(threads / G) * 2 * max_l * sizeof(uint16_t);
    const int64_t items = a.end - a.begin;
    const int grid = grid_for(items * G, threads, 16);
    auto kern = write_pass ? expand_tile<G, WPL, true> : expand_tile<G, WPL, false>;
    if (smem > 48 * 1024) MCE_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    kern<<<grid, threads, smem, s>>>(a, max_l);
    MCE_LAUNCH_CHECK();
}

}  // namespace

void launch_build_adj(const RootInfo *roots, int64_t nroots, int W, const int64_t *orp, const int32_t *ocol,
                      uint64_t *adj, int64_t adj_words, cudaStream_t s, unsigned long long *bytes) {
    if (nroots <= 0) return;
    if (W == 1) {
        build_adj_w1<<<grid_for(nroots * 32, 256, 16), 256, 0, s>>>(roots, nroots, orp, ocol, adj);
    } else {
        // shared-memory bit matrix up to W = 16 (L <= 1024: 128 KB), the
        // staged V, and the span bit map + word ranks (48 KB)
        const int64_t Lmax = 64ll * W;
        const size_t map_bytes = (size_t)kSpanWords * 4 + (size_t)kSpanWords * 2;
        const size_t base = sizeof(int32_t) * (size_t)((Lmax + 3) & ~3ll);
        if (W <= 16) {
            const size_t smem = base + (size_t)Lmax * W * 8 + map_bytes;
            static size_t attr_set = 0;
            if (attr_set < smem) {
                MCE_CUDA(cudaFuncSetAttribute(build_adj_block<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                              (int)smem));
                attr_set = smem;
            }
            build_adj_block<true><<<grid_for(nroots, 1, 8), 1024, smem, s>>>(roots, nroots, W, orp, ocol, adj,
                                                                              (int)Lmax, 1, bytes);
        } else {
            const size_t smem = base + map_bytes;
            static size_t attr_set = 0;
            if (attr_set < smem) {
                MCE_CUDA(cudaFuncSetAttribute(build_adj_block<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                              (int)smem));
                attr_set = smem;
            }
            MCE_CUDA(cudaMemsetAsync(adj, 0, sizeof(uint64_t) * (size_t)adj_words, s));
            build_adj_block<false><<<grid_for(nroots, 1, 8), 1024, smem, s>>>(roots, nroots, W, orp, ocol, adj,
                                                                               (int)Lmax, 1, bytes);
        }
    }
    MCE_LAUNCH_CHECK();
}

void launch_init_level1(const RootInfo *roots, int64_t nroots, int W, uint64_t *P, int32_t *slot, int32_t *parent,
                        int32_t *vloc, cudaStream_t s) {
    if (nroots <= 0) return;
    init_level1_kernel<<<grid_for(nroots, 256), 256, 0, s>>>(roots, nroots, W, P, slot, parent, vloc);
    MCE_LAUNCH_CHECK();
}

template <int W>
void launch_thread(const ExpandArgs &a, bool write_pass, cudaStream_t s) {
    const int grid = grid_for(a.end - a.begin, 256, 8);
    if (write_pass)
        expand_thread<W, true><<<grid, 256, 0, s>>>(a);
    else
        expand_thread<W, false><<<grid, 256, 0, s>>>(a);
    MCE_LAUNCH_CHECK();
}

template <int G>
void launch_lock(const ExpandArgs &a0, cudaStream_t s) {
    constexpr int threads = 512;
    ExpandArgs a = a0;
    const int64_t n = a.end - a.begin;
    const size_t smem = (size_t)64 * G * G * 8 + (size_t)(threads / G) * 64 * G * 2;
    static int per_sm = 0;
    if (!per_sm) {
        MCE_CUDA(cudaFuncSetAttribute(expand_lock<G>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, expand_lock<G>, threads, smem));
        per_sm = std::max(per_sm, 1);
    }
    const int64_t slots = (int64_t)num_sms() * per_sm;
    // ~8 chunks per resident block (dynamic balance), at most 16 candidates per tile; a
    // small level (one entry per root at k = 1) takes chunks of one entry, spread over SMs
    a.chunk = (int32_t)std::max<int64_t>(1, std::min<int64_t>(16 * (threads / G), ceil_div(n, 8 * slots)));
    MCE_CUDA(cudaMemsetAsync(a.chunk_ctr, 0, sizeof(unsigned long long), s));
    const int64_t nchunks = ceil_div(n, a.chunk);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(nchunks, slots));
    expand_lock<G><<<grid, threads, smem, s>>>(a, nchunks);
    MCE_LAUNCH_CHECK();
}

template <int G, int WPL>
void launch_wide(const ExpandArgs &a0, cudaStream_t s) {
    constexpr int threads = 256, W = G * WPL;
    ExpandArgs a = a0;
    const int64_t n = a.end - a.begin;
    static int per_sm = 0;
    if (!per_sm) {
        MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, expand_wide<G, WPL>, threads, 0));
        per_sm = std::max(per_sm, 1);
    }
    const int64_t slots = (int64_t)num_sms() * per_sm;
    // per-warp chunks: T candidates (one trip) or a few trips when the level is large
    const int64_t warps = slots * (threads / 32);
    a.chunk = (int32_t)((32 / G) * std::max<int64_t>(1, std::min<int64_t>(4, n / (warps * 8 * (32 / G)))));
    MCE_CUDA(cudaMemsetAsync(a.chunk_ctr, 0, sizeof(unsigned long long), s));
    const int64_t nchunks = ceil_div(n, a.chunk);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(nchunks, slots));
    // per-tile colouring orders (64 W u16 each) in the caller's scratch: at most as many blocks as it holds
    const int64_t per_block = (int64_t)(threads / G) * 64 * W;
    const int g2 = (int)std::min<int64_t>(grid, a.wscratch_n / per_block);
    if (g2 < 1) fail(4, "wide expansion: scratch below one block's colouring orders");
    expand_wide<G, WPL><<<g2, threads, 0, s>>>(a, nchunks, a.wscratch);
    MCE_LAUNCH_CHECK();
}

static int wide_kind() {  // lanes per candidate for the wide pass (MCE_WIDE_G = 8 / 16 / 32; 0 = off)
    static int g = -1;
    if (g < 0) {
        const char *e = getenv("MCE_WIDE_G");
        g = e ? atoi(e) : 16;
    }
    return g;
}

int wide_min_w() {  // narrowest level the wide pass takes (MCE_WIDE_MIN_W; default 32 words)
    static int w = -1;
    if (w < 0) {
        const char *e = getenv("MCE_WIDE_MIN_W");
        w = e ? atoi(e) : 32;
        if (wide_kind() <= 0) w = 1 << 30;
    }
    return w;
}

void launch_expand(const ExpandArgs &a, bool write_pass, cudaStream_t s) {
    const int64_t items = a.end - a.begin;
    if (items <= 0) return;
    if (!write_pass && !a.perm && a.wscratch && a.Wp >= wide_min_w() && a.Wp <= 64) {
        const int g = wide_kind();
        switch (a.Wp) {
            case 4: return launch_wide<4, 1>(a, s);
            case 8: return g == 4 ? launch_wide<4, 2>(a, s) : launch_wide<8, 1>(a, s);
            case 16: return g == 8 ? launch_wide<8, 2>(a, s) : launch_wide<16, 1>(a, s);
            case 32: return g == 8 ? launch_wide<8, 4>(a, s) : (g == 32 ? launch_wide<32, 1>(a, s) : launch_wide<16, 2>(a, s));
            case 64: return g == 8 ? launch_wide<8, 8>(a, s) : (g == 32 ? launch_wide<32, 2>(a, s) : launch_wide<16, 4>(a, s));
            default: break;
        }
    }
    if (!write_pass && a.perm) {  // shared-memory count pass (the caller grouped the level by slot)
        if (a.Wp == 4) return launch_lock<4>(a, s);
        if (a.Wp == 8) return launch_lock<8>(a, s);
        if (a.Wp == 16) return launch_lock<16>(a, s);
        fail(1, "internal: shared-memory expansion for an unsupported width");
    }
    if (a.Wp == 1) {
        launch_thread<1>(a, write_pass, s);
    } else if (a.Wp == 2) {
        launch_thread<2>(a, write_pass, s);
    } else if (a.Wp == 4) {
        launch_thread<4>(a, write_pass, s);
    } else if (a.Wp <= 32) {
        // a whole warp per candidate: 8- and 16-lane tiles (four or two
        // candidates per warp) measured slower on dense800 (66 -> 99 ms count
        // pass): the tiles of a warp diverge between colouring and branching
        launch_tile<32, 1>(a, write_pass, s);
    } else if (a.Wp <= 64) {
        launch_tile<32, 2>(a, write_pass, s);
    } else if (a.Wp <= 128) {
        launch_tile<32, 4>(a, write_pass, s);
    } else {
        launch_tile<32, 8>(a, write_pass, s);
    }
}

void launch_group_by_slot(const int32_t *slot, int64_t n, int32_t nslots, int32_t *hist, int64_t *offs,
                          int64_t *scan_tmp, int32_t *perm, cudaStream_t s) {
    if (n <= 0) return;
    MCE_CUDA(cudaMemsetAsync(hist, 0, sizeof(int32_t) * std::max<int32_t>(nslots, 1), s));
    slot_hist_kernel<<<grid_for(n, 256), 256, 0, s>>>(slot, n, hist);
    MCE_LAUNCH_CHECK();
    exclusive_scan_i32(hist, offs, nslots, scan_tmp, s);
    slot_scatter_kernel<<<grid_for(n, 256), 256, 0, s>>>(slot, n, reinterpret_cast<unsigned long long *>(offs),
                                                          perm);
    MCE_LAUNCH_CHECK();
}

void launch_reroot_sizes(const uint64_t *P, int Ps, int W, int64_t n, int32_t *Lp, int32_t *cls, int64_t *hist,
                         cudaStream_t s) {
    if (n <= 0) return;
    reroot_sizes_kernel<<<grid_for(n, 256), 256, 0, s>>>(P, Ps, W, n, Lp, cls, reinterpret_cast<unsigned long long *>(hist));
    MCE_LAUNCH_CHECK();
}
void launch_gather_i32(const int32_t *src, const int32_t *idx, int64_t n, int32_t *dst, cudaStream_t s) {
    if (n <= 0) return;
    gather_i32_kernel<<<grid_for(n, 256), 256, 0, s>>>(src, idx, n, dst);
    MCE_LAUNCH_CHECK();
}
void launch_reroot_build(const ExpandArgs &a, const int32_t *list, int64_t cnt, const int64_t *voff, int Wn,
                         int32_t *nV, uint64_t *nA, RootInfo *nroots, uint64_t *nP, int32_t *nslot, int32_t *nparent,
                         int32_t *nvloc, int32_t *nprefix, cudaStream_t s) {
    if (cnt <= 0) return;
    if (Wn > kRerootMaxL / 64) fail(1, "internal: re-rooted space wider than 16 words");
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(cnt, kRerootWarps), (int64_t)num_sms() * 8));
    reroot_build_kernel<<<grid, 32 * kRerootWarps, 0, s>>>(a, list, cnt, voff, Wn, nV, nA, nroots, nP, nslot, nparent,
                                                            nvloc, nprefix);
    MCE_LAUNCH_CHECK();
}

void launch_materialize_pairs(const ExpandArgs &a, int64_t n, cudaStream_t s) {
    if (n <= 0) return;
    materialize_pairs_kernel<<<(int)std::min<int64_t>(n, (int64_t)num_sms() * 8), kMatThreads, 0, s>>>(a, n);
    MCE_LAUNCH_CHECK();
}

void launch_expand_small(const ExpandArgs &a, uint8_t *scratch, int64_t scratch_bytes, SmallOut *out,
                         LevelLink *chain, cudaStream_t s) {
    expand_small<<<1, kSmallThreads, 0, s>>>(a, scratch, scratch_bytes, out, chain);
    MCE_LAUNCH_CHECK();
}

void launch_shard_flags(const ExpandArgs &a, int64_t n, int32_t k, int32_t rank, int32_t count, int32_t *flag,
                        cudaStream_t s) {
    if (n <= 0) return;
    shard_flags_kernel<<<grid_for(n, 256), 256, 0, s>>>(a, n, k, rank, count, flag);
    MCE_LAUNCH_CHECK();
}
void launch_gather_level(int64_t n, const int32_t *flag, const int64_t *pos, int W, int Ps, const uint64_t *P,
                         const int32_t *slot, const int32_t *parent, const int32_t *vloc, uint64_t *oP,
                         int32_t *oslot, int32_t *oparent, int32_t *ovloc, cudaStream_t s) {
    if (n <= 0) return;
    gather_level_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, flag, pos, W, Ps, P, slot, parent, vloc, oP, oslot,
                                                          oparent, ovloc);
    MCE_LAUNCH_CHECK();
}
void launch_classify_roots(int64_t n, const int64_t *orp, int32_t min_len, int32_t shard_rank, int32_t shard_count,
                           const uint8_t *keep, int64_t keep_T, int32_t *cls, int64_t *hist, cudaStream_t s) {
    classify_roots_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, orp, min_len, shard_rank, shard_count, keep, keep_T,
                                                           cls, (unsigned long long *)hist);
    MCE_LAUNCH_CHECK();
}
void launch_find_window(const int64_t *prefix, int64_t hi, int64_t lo_min, int64_t room, int64_t row_bytes,
                        int64_t per_root, int64_t *out, cudaStream_t s) {
    find_window_kernel<<<1, 1, 0, s>>>(prefix, hi, lo_min, room, row_bytes, per_root, out);
    MCE_LAUNCH_CHECK();
}
void launch_flag_eq(int64_t n, const int32_t *cls, int32_t c, int32_t *flag, cudaStream_t s) {
    flag_eq_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, cls, c, flag);
    MCE_LAUNCH_CHECK();
}
void launch_compact(int64_t n, const int32_t *flag, const int64_t *pos, int32_t *out, cudaStream_t s) {
    compact_idx_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, flag, pos, out);
    MCE_LAUNCH_CHECK();
}
void launch_make_roots(const int32_t *list, int64_t count, int64_t stride, int W, const int64_t *orp,
                       const int64_t *row_prefix, RootInfo *roots, cudaStream_t s) {
    if (count <= 0) return;
    make_roots_kernel<<<grid_for(count, 256), 256, 0, s>>>(list, count, stride, W, orp, row_prefix, roots);
    MCE_LAUNCH_CHECK();
}
void launch_root_lengths(const int32_t *list, int64_t count, int64_t stride, const int64_t *orp, int32_t *len,
                         cudaStream_t s) {
    if (count <= 0) return;
    root_lengths_kernel<<<grid_for(count, 256), 256, 0, s>>>(list, count, stride, orp, len);
    MCE_LAUNCH_CHECK();
}
void launch_find_chunk_end(const int64_t *offsets, int64_t a, int64_t n, int64_t cap, int64_t *out,
                           cudaStream_t s) {
    find_chunk_end_kernel<<<1, 1, 0, s>>>(offsets, a, n, cap, out);
    MCE_LAUNCH_CHECK();
}

}  // namespace mce
