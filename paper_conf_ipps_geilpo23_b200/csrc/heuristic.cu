// Greedy lower bound on omega (PAPER.md IV-A, lines 103-109, Algorithm 1).
//
// Multi-run: the h vertices with the highest threshold (degree or core
// number) each seed one run; a run holds C = {seed}, P = N(seed) and
// repeatedly adds the candidate with the highest threshold (ties: smaller id,
// the first maximum of an id-sorted segment = Algorithm 1 line 34's segmented
// max), then keeps only the candidates adjacent to it (lines 35-38).  The
// single-run variants are the h = 1 case (the first pick from "all vertices"
// is the top vertex).
//
// B200 mapping: one warp per run instead of Algorithm 1's segmented
// CUB passes -- the argmax is a warp max-reduction over a 64-bit key
// (threshold << 32 | ~id), the filter is a warp-cooperative membership test
// (binary search in the sorted adjacency list of the added vertex) compacted
// in place with __ballot_sync/__popc, so every run stays in one warp's
// registers + one contiguous scratch segment and no host round trip is needed
// per iteration.
#include <cub/device/device_radix_sort.cuh>

#include <algorithm>
#include <vector>

#include "graph.cuh"
#include "heuristic.cuh"
#include "mce.h"

namespace mce {

namespace {

__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        unsigned long long y = __shfl_xor_sync(0xffffffffu, x, o);
        x = y > x ? y : x;
    }
    return x;
}

__device__ __forceinline__ unsigned long long pick_key(const int32_t *__restrict__ thr, int32_t x) {
    return ((unsigned long long)(uint32_t)__ldg(thr + x) << 32) | (unsigned long long)(0x7fffffffu - (uint32_t)x);
}

// x ~ w?  Binary search for x in w's sorted adjacency list.  Every lane of a
// run searches the SAME list N(w) (w is the pick, the highest-threshold
// candidate, so for the degree heuristic its list is the longest of all): the
// top levels of the search tree are shared by all lanes and candidates (L1
// hits), and P is kept in id order, so neighbouring lanes end in neighbouring
// sectors.  Searching each candidate's own (shorter) list instead costs two
// rowptr loads and ~log2(deg x) probes into a different cold list per
// candidate (measured on rmat22: 44 GB of DRAM reads for the heuristic runs).
#ifndef HEUR_SEARCH_W
#define HEUR_SEARCH_W 1
#endif
__device__ __forceinline__ bool adjacent(const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                         int32_t x, int32_t w, int64_t wb, int64_t we) {
#if HEUR_SEARCH_W
    return contains_sorted(col, wb, we, x);
#else
    const int64_t xb = __ldg(rowptr + x), xe = __ldg(rowptr + x + 1);
    if (xe - xb < we - wb) return contains_sorted(col, xb, xe, w);
    return contains_sorted(col, wb, we, x);
#endif
}

// Early abort (exact).  A run's final size is at most |C| + |P| at any
// point, and at most t(s) + 1 from the start, t(s) = min(deg(s), core(s)) (a
// clique through s has at most core(s) + 1 vertices).  Unless every run size
// is wanted, a run stops as soon as that cap falls STRICTLY below the best
// size found so far: it can no longer reach the best, so neither the best
// size nor the winning seed (the first in seed order among runs reaching it)
// changes.  The size it stores is then < the final best, never equal.
__device__ __forceinline__ int32_t ld_best(const int32_t *best) {
    int32_t v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(best) : "memory");
    return v;
}

// Candidate filter (exact, with the early abort).  A candidate x whose
// threshold (degree, or core number: both bound the size of any clique
// through x by thr(x) + 1) is below best - 1 can never be picked by a run that
// still reaches best: picks go by the highest threshold, so x is picked only
// once every candidate above it is gone, and the clique then holds x, hence
// has at most thr(x) + 1 < best vertices.  Dropping such candidates therefore
// changes neither the picks of any run that reaches best (so neither the best
// size nor the winning seed nor its clique) nor whether a run reaches it;
// |C| + |P| then counts only candidates that can matter, so hopeless runs
// abort sooner, and the adjacency tests of the dropped candidates (most of a
// power-law seed's neighbours) are never made.  b == 0 (every run size
// wanted, Algorithm 1 verbatim) keeps every candidate.
#ifndef HEUR_FILTER
#define HEUR_FILTER 1
#endif
__device__ __forceinline__ bool useful(const int32_t *__restrict__ thr, int32_t x, int32_t b,
                                       const int32_t *__restrict__ core = nullptr) {
    return !HEUR_FILTER || b <= 1 || (__ldg(thr + x) + 1 >= b && (!core || __ldg(core + x) + 1 >= b));
}

// Hub bit matrix (exact acceleration of the runs on power-law graphs).  H =
// the highest-degree vertices (whole degree buckets, at most kHubBig of them),
// indexed so that the (at most kHubTail) highest come first; M = their induced
// adjacency, K rows of KW words; hkey = their pick keys.
//  * adjacency tests between two hubs are one bit of M instead of a binary
//    search (rmat22: the 110K vertices of degree >= omega - 1 are all hubs, so
//    once the candidate filter has run every test of every run is a bit load);
//  * once every candidate of a run is among the first KT hubs (the tail set),
//    the run continues on a bit set over them: the pick is a max over the set
//    bits' keys, the filter one AND with M's row prefix.
// Same picks, same sizes as the list form (the key encodes threshold and id).
#ifndef HUB_BIG
#define HUB_BIG 131072
#endif
constexpr int kHubBig = HUB_BIG;          // lookup matrix: at most 2^17 rows of 2^11 words (2 GiB)
#ifndef HUB_TAIL
#define HUB_TAIL 2048  // measured 2048 / 4096 / 8192 / 16384 / 32768: rmat22 43.4 / 44.5 / 44.3 / 49.5 / 58.0 ms (one word per lane)
#endif
constexpr int kHubTail = HUB_TAIL;        // bit-set tail: the first kHubTail hubs
#ifndef HUB_ROWS
#define HUB_ROWS 16384  // rmat22: 4096 / 16384 / 131072 (every hub) rows = 35.5 / 35.4 / 36.3 ms per step
#endif
constexpr int kHubRows = HUB_ROWS;        // hubs with a matrix row (the rest: columns only)
constexpr int kHubWords = kHubTail / 64;  // 128
constexpr int kHubWPL = kHubWords / 32;   // words per lane
struct Hub {
    const int32_t *hid = nullptr;              // [n] hub index or -1
    const int32_t *hv = nullptr;               // [K] hub -> vertex
    const unsigned long long *hkey = nullptr;  // [K] pick keys
    const uint64_t *M = nullptr;               // [K][KW]
    int K = 0, KW = 0, KT = 0;                 // KT: hubs of the tail set (indices < KT), <= kHubTail
    int KR = 0;                                // hubs with a matrix row (indices < KR, the highest degrees)
};

// The rest of a run whose candidates are all hubs, by one warp: P = the
// list src[0..len) (all in H) becomes a bit set; returns the final size.
__device__ int32_t hub_tail_warp(const Hub &H, const int32_t *src, int64_t len, int32_t csize, int32_t *clique,
                                 const int32_t *best) {
    const int lane = threadIdx.x & 31;
    uint64_t P[kHubWPL];
#pragma unroll
    for (int t = 0; t < kHubWPL; ++t) P[t] = 0;
    // build: lane l collects the members whose word is owned by l (word % 32 == l)
    for (int64_t i0 = 0; i0 < len; i0 += 32) {
        const int64_t i = i0 + lane;
        const int h = i < len ? __ldg(H.hid + src[i]) : -1;  // < KT for every member (caller)
        for (int src_lane = 0; src_lane < 32; ++src_lane) {
            const int hh = __shfl_sync(0xffffffffu, h, src_lane);
            if (hh >= 0 && ((hh >> 6) & 31) == lane) {
#pragma unroll
                for (int t = 0; t < kHubWPL; ++t)
                    if (t == (hh >> 11)) P[t] |= 1ull << (hh & 63);
            }
        }
    }
    while (true) {
        int pc = 0;
#pragma unroll
        for (int t = 0; t < kHubWPL; ++t) pc += __popcll(P[t]);
        pc = __reduce_add_sync(0xffffffffu, pc);
        if (pc == 0) break;
        if (best) {
            int32_t b = 0;
            if (lane == 0) b = ld_best(best);
            b = __shfl_sync(0xffffffffu, b, 0);
            if (csize + pc < b) break;
        }
        unsigned long long key = 0;
        int hb = -1;
#pragma unroll
        for (int t = 0; t < kHubWPL; ++t) {
            uint64_t q = P[t];
            while (q) {
                const int b = __ffsll((long long)q) - 1;
                q &= q - 1;
                const int h = ((t * 32 + lane) << 6) + b;
                const unsigned long long k2 = __ldg(H.hkey + h);
                if (k2 > key) {
                    key = k2;
                    hb = h;
                }
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long y = __shfl_xor_sync(0xffffffffu, key, o);
            const int yh = __shfl_xor_sync(0xffffffffu, hb, o);
            if (y > key) {
                key = y;
                hb = yh;
            }
        }
        if (clique && lane == 0) clique[csize] = (int32_t)(0x7fffffffu - (uint32_t)(key & 0xffffffffull));
        ++csize;
        const uint64_t *row = H.M + (int64_t)hb * H.KW;
        const int tw = (H.KT + 63) >> 6;  // words of the tail set
#pragma unroll
        for (int t = 0; t < kHubWPL; ++t) {
            const int w = t * 32 + lane;
            P[t] &= w < tw ? __ldg(row + w) : 0ull;
            if (w == (hb >> 6)) P[t] &= ~(1ull << (hb & 63));
        }
    }
    return csize;
}

// x ~ w with the hub bit matrix when both are hubs (hw = hid[w] or -1);
// also reports whether x is in the tail set
__device__ __forceinline__ bool adjacent_h(const Hub &H, int hw, const int64_t *__restrict__ rowptr,
                                           const int32_t *__restrict__ col, int32_t x, int32_t w, int64_t wb,
                                           int64_t we, bool &x_hub) {
    if (H.K) {
        const int hx = __ldg(H.hid + x);
        x_hub = hx >= 0 && hx < H.KT;
        if (hx >= 0 && hw >= 0 && hw < H.KR) return (__ldg(H.M + (int64_t)hw * H.KW + (hx >> 6)) >> (hx & 63)) & 1ull;
    } else {
        x_hub = false;
    }
    return adjacent(rowptr, col, x, w, wb, we);
}

// One greedy run for seed s by a tile of G lanes (G = 8 or 32) of the calling
// warp.  Returns the clique size (a partial size < the best when aborted).
template <int G>
__device__ int32_t greedy_run(int32_t s, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                              const int32_t *__restrict__ thr, int32_t *__restrict__ scratch, const int32_t *best,
                              const Hub &H, const int32_t *__restrict__ fcore = nullptr) {
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1);
    const int gbase = lane & ~(G - 1);
    const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
    const int64_t base = rowptr[s];
    int64_t len = rowptr[s + 1] - base;
    const int32_t *src = col + base;  // first round reads the CSR row directly
    int32_t *buf = scratch + base;    // later rounds work in place in the seed's segment
    int32_t csize = 1;
    while (len > 0) {
        int32_t b = 0;  // current best (0: no abort, no candidate filter)
        if (best) {
            if (gl == 0) b = ld_best(best);
            b = __shfl_sync(gmask, b, 0, G);
            if (csize + len < b) break;
        }
        unsigned long long key = 0;
        for (int64_t i = gl; i < len; i += G) {
            unsigned long long k2 = pick_key(thr, src[i]);
            key = k2 > key ? k2 : key;
        }
#pragma unroll
        for (int o = G / 2; o > 0; o >>= 1) {
            unsigned long long y = __shfl_xor_sync(gmask, key, o, G);
            key = y > key ? y : key;
        }
        const int32_t w = (int32_t)(0x7fffffffu - (uint32_t)(key & 0xffffffffull));
        ++csize;
        const int64_t wb = rowptr[w], we = rowptr[w + 1];
        const int hw = H.K ? __ldg(H.hid + w) : -1;
        int64_t out = 0;
        int nonhub = 0;
        for (int64_t i0 = 0; i0 < len; i0 += G) {
            int64_t i = i0 + gl;
            int32_t x = i < len ? src[i] : -1;
            bool xh = true;
            bool keep = i < len && x != w && useful(thr, x, b, fcore) && adjacent_h(H, hw, rowptr, col, x, w, wb, we, xh);
            const unsigned m = (__ballot_sync(gmask, keep) & gmask) >> gbase;
            if (keep) buf[out + __popc(m & ((1u << gl) - 1u))] = x;
            out += __popc(m);
            if (G == 32 && H.K) nonhub += __popc(__ballot_sync(gmask, keep && !xh));
        }
        __syncwarp(gmask);
        src = buf;
        len = out;
        if (G == 32 && H.K && len > 0 && nonhub == 0) return hub_tail_warp(H, src, len, csize, nullptr, best);
    }
    return csize;
}

// One greedy run for seed s by the whole block (NT threads): block-wide argmax
// and an order-preserving in-place compaction.  Hub seeds (degree > kBigSeed)
// run this way so a long run is not serialised on one warp; the replay of the
// winning run uses it too, writing the clique (in order added).
#ifndef BLOCK_RUN
#define BLOCK_RUN 256  // rmat22, round 2: 256 / 512 / 1024 threads = 37.5 / 37.8 / 40.6 ms per step (round 1, before the candidate filter: 95.4 / 81.8 / 90.7)
#endif
constexpr int kBlockRun = BLOCK_RUN;
constexpr int64_t kBigSeed = 1024;
template <int NT>
__device__ int32_t block_run(int32_t s, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                             const int32_t *__restrict__ thr, int32_t *__restrict__ scratch, int32_t *clique,
                             const int32_t *best, const Hub &H, const int32_t *__restrict__ fcore = nullptr) {
    __shared__ unsigned long long wkey[NT / 32];
    __shared__ int32_t wcnt[NT / 32], wnon[NT / 32];
    __shared__ int32_t sbest, sres;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int64_t base = rowptr[s];
    int64_t len = rowptr[s + 1] - base;
    const int32_t *src = col + base;
    int32_t *buf = scratch + base;
    int32_t csize = 1;
    if (clique && threadIdx.x == 0) clique[0] = s;
    while (len > 0) {
        int32_t b = 0;  // current best (0: no abort, no candidate filter)
        if (best) {
            if (threadIdx.x == 0) sbest = ld_best(best);
            __syncthreads();
            b = sbest;
            __syncthreads();
            if (csize + len < b) break;
        }
        unsigned long long key = 0;
        for (int64_t i = threadIdx.x; i < len; i += NT) {
            const unsigned long long k2 = pick_key(thr, src[i]);
            key = k2 > key ? k2 : key;
        }
        key = warp_max_u64(key);
        if (lane == 0) wkey[wid] = key;
        __syncthreads();
        if (wid == 0) {
            key = warp_max_u64(lane < NT / 32 ? wkey[lane] : 0ull);
            if (lane == 0) wkey[0] = key;
        }
        __syncthreads();
        key = wkey[0];
        const int32_t w = (int32_t)(0x7fffffffu - (uint32_t)(key & 0xffffffffull));
        if (clique && threadIdx.x == 0) clique[csize] = w;
        ++csize;
        const int64_t wb = rowptr[w], we = rowptr[w + 1];
        const int hw = H.K ? __ldg(H.hid + w) : -1;
        int64_t out = 0;
        int32_t nonhub = 0;
        for (int64_t i0 = 0; i0 < len; i0 += NT) {
            const int64_t i = i0 + threadIdx.x;
            const int32_t x = i < len ? src[i] : -1;
            bool xh = true;
            const bool keep = i < len && x != w && useful(thr, x, b, fcore) && adjacent_h(H, hw, rowptr, col, x, w, wb, we, xh);
            const unsigned m = __ballot_sync(0xffffffffu, keep);
            const unsigned nh = H.K ? __ballot_sync(0xffffffffu, keep && !xh) : 0u;
            __syncthreads();  // wkey/wcnt reuse, and every read of this chunk precedes its writes
            if (lane == 0) {
                wcnt[wid] = __popc(m);
                wnon[wid] = __popc(nh);
            }
            __syncthreads();
            int32_t before = 0, total = 0;
#pragma unroll
            for (int j = 0; j < NT / 32; ++j) {
                const int32_t c = wcnt[j];
                before += j < wid ? c : 0;
                total += c;
                nonhub += wnon[j];
            }
            if (keep) buf[out + before + __popc(m & lanemask_lt())] = x;
            out += total;
        }
        __syncthreads();
        src = buf;
        len = out;
        if (H.K && len > 0 && nonhub == 0) {  // the rest on a bit set over the hubs, by warp 0
            if (wid == 0) {
                const int32_t c = hub_tail_warp(H, src, len, csize, clique, best);
                if (lane == 0) sres = c;
            }
            __syncthreads();
            csize = sres;
            __syncthreads();
            return csize;
        }
    }
    return csize;
}

// cap t(s) + 1 on the size of any run from seed s (see ld_best)
__device__ __forceinline__ int64_t seed_cap(int32_t s, const int64_t *__restrict__ rowptr,
                                            const int32_t *__restrict__ core) {
    int64_t c = rowptr[s + 1] - rowptr[s];
    if (core) c = min(c, (int64_t)__ldg(core + s));
    return c + 1;
}

// Hub seeds (degree > kBigSeed): one block per run, launched before the rest
// so the long runs start first and their sizes prune the short ones.
__global__ void __launch_bounds__(kBlockRun) greedy_big_kernel(int64_t nbig, const int32_t *__restrict__ big,
                                                               const int64_t *__restrict__ rowptr,
                                                               const int32_t *__restrict__ col,
                                                               const int32_t *__restrict__ thr,
                                                               const int32_t *__restrict__ core,
                                                               int32_t *__restrict__ scratch,
                                                               int32_t *__restrict__ run_size, int32_t *best_size,
                                                               int abort_runs, const Hub H) {
    for (int64_t i = blockIdx.x; i < nbig; i += gridDim.x) {
        const int32_t s = big[i];
        int32_t c = 1;
        if (!abort_runs || seed_cap(s, rowptr, core) >= ld_best(best_size))
            c = block_run<kBlockRun>(s, rowptr, col, thr, scratch, nullptr, abort_runs ? best_size : nullptr, H,
                                     abort_runs ? core : nullptr);
        if (threadIdx.x == 0) {
            run_size[s] = c;
            atomicMax(best_size, c);
        }
        __syncthreads();
    }
}

// The other seeds (degree <= kBigSeed).  Warp w takes seeds [4w, 4w+4): when
// all four have degree <= 64 they run in parallel on 8-lane tiles (low-degree
// seeds leave most of a warp idle), otherwise one after another on the whole
// warp.  A warp publishes its best with one atomicMax per group of seeds, so
// later runs abort against it.  (A thread per short seed was measured 2x
// slower: its candidate rows and adjacency searches are 32 separate streams.)
__global__ void __launch_bounds__(256) greedy_kernel(int64_t nseeds, const int32_t *__restrict__ seeds,
                                                     const int64_t *__restrict__ rowptr,
                                                     const int32_t *__restrict__ col, const int32_t *__restrict__ thr,
                                                     const int32_t *__restrict__ core,
                                                     int32_t *__restrict__ scratch, int32_t *__restrict__ run_size,
                                                     int32_t *best_size, int abort_runs, const Hub H) {
    const Hub none{};
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    const int32_t *best = abort_runs ? best_size : nullptr;
    int32_t published = 0;
    for (int64_t i0 = warp * 4; i0 < nseeds; i0 += nwarps * 4) {
        const int64_t my = i0 + (lane >> 3);
        int32_t s_mine = my < nseeds ? seeds[my] : -1;
        int64_t d_mine = s_mine >= 0 ? rowptr[s_mine + 1] - rowptr[s_mine] : 0;
        if (d_mine > kBigSeed) s_mine = -1;  // run by greedy_big_kernel
        if (s_mine >= 0 && best && seed_cap(s_mine, rowptr, core) < ld_best(best_size)) {
            if ((lane & 7) == 0) run_size[s_mine] = 1;  // cannot reach the best: not run
            s_mine = -1;
        }
        if (s_mine < 0) d_mine = 0;
        int32_t mybest = 0;
        if (!__ballot_sync(0xffffffffu, s_mine >= 0)) continue;
        if (__all_sync(0xffffffffu, d_mine <= 64)) {
            if (s_mine >= 0) {
                const int32_t c = greedy_run<8>(s_mine, rowptr, col, thr, scratch, best, none, best ? core : nullptr);
                if ((lane & 7) == 0) run_size[s_mine] = c;
                mybest = c;
            }
        } else {
            for (int t = 0; t < 4; ++t) {
                const int32_t s = __shfl_sync(0xffffffffu, s_mine, 8 * t);
                if (s < 0) continue;
                const int32_t c = greedy_run<32>(s, rowptr, col, thr, scratch, best, H, best ? core : nullptr);
                if (lane == 0) run_size[s] = c;
                mybest = max(mybest, c);
            }
        }
        mybest = __reduce_max_sync(0xffffffffu, mybest);
        if (lane == 0 && mybest > published) {
            atomicMax(best_size, mybest);
            published = mybest;
        }
        __syncwarp();
    }
}

__global__ void big_flags_kernel(int64_t nseeds, const int32_t *__restrict__ seeds,
                                 const int64_t *__restrict__ rowptr, int32_t *flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nseeds; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t s = seeds[i];
        flag[i] = rowptr[s + 1] - rowptr[s] > kBigSeed;
    }
}

__global__ void seed_degree_kernel(int64_t nbig, const int32_t *__restrict__ big, const int64_t *__restrict__ rowptr,
                                   int32_t *deg) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nbig; i += (int64_t)gridDim.x * blockDim.x)
        deg[i] = (int32_t)(rowptr[big[i] + 1] - rowptr[big[i]]);
}

__global__ void gather_flagged_kernel(int64_t n, const int32_t *__restrict__ in, const int32_t *__restrict__ flag,
                                      const int64_t *__restrict__ pos, int32_t *out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (flag[i]) out[pos[i]] = in[i];
}

// among seeds whose run reached best, the first in seed order (threshold desc, id asc)
__global__ void best_seed_kernel(int64_t nseeds, const int32_t *__restrict__ seeds, const int32_t *__restrict__ thr,
                                 const int32_t *__restrict__ run_size, const int32_t *best_size,
                                 unsigned long long *best_key) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nseeds; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t s = seeds[i];
        if (run_size[s] == *best_size) atomicMax(best_key, pick_key(thr, s));
    }
}

// Replay of the winning run to recover its clique (one block, nothing else running)
constexpr int kReplay = 1024;
__global__ void __launch_bounds__(kReplay) replay_kernel(const unsigned long long *best_key, const int32_t *best,
                                                         const int32_t *__restrict__ core,
                                                         const int64_t *__restrict__ rowptr,
                                                         const int32_t *__restrict__ col,
                                                         const int32_t *__restrict__ thr,
                                                         int32_t *__restrict__ scratch, int32_t *clique, const Hub H) {
    const int32_t s = (int32_t)(0x7fffffffu - (uint32_t)(*best_key & 0xffffffffull));
    // the winning run reaches *best, so the filter (and the abort) against it
    // leaves its picks unchanged (see useful())
    block_run<kReplay>(s, rowptr, col, thr, scratch, clique, best, H, core);
}

__global__ void degree_thr_kernel(int64_t n, const int64_t *__restrict__ rowptr, int32_t *thr) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        thr[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
}

__global__ void thr_hist_kernel(int64_t n, const int32_t *__restrict__ thr, int64_t *bins) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        atomicAdd((unsigned long long *)(bins + thr[v]), 1ull);
}

__global__ void tie_flags_kernel(int64_t n, const int32_t *__restrict__ thr, int32_t tau, int32_t *flag) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        flag[v] = thr[v] == tau;
}

// seed flag = thr > tau, or thr == tau and among the first `quota` ties by id
__global__ void seed_flags_kernel(int64_t n, const int32_t *__restrict__ thr, int32_t tau,
                                  const int64_t *__restrict__ tie_rank, int64_t quota, int32_t *flag) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        flag[v] = thr[v] > tau || (thr[v] == tau && tie_rank[v] < quota);
}

__global__ void compact_kernel(int64_t n, const int32_t *__restrict__ flag, const int64_t *__restrict__ pos,
                               int32_t *out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        if (flag[v]) out[pos[v]] = (int32_t)v;
}

__global__ void strided_gather_kernel(const int32_t *__restrict__ in, int64_t count, int64_t stride, int32_t *out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = in[i * stride];
}

__global__ void iota_kernel(int64_t n, int32_t *out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        out[v] = (int32_t)v;
}

// degree bucket: 4 mantissa bits below the leading one (monotone in d)
__device__ __forceinline__ int deg_bucket(int64_t d) {
    if (d <= 0) return 0;
    const int e = 63 - __clzll((long long)d);
    const int m = e >= 4 ? (int)((d >> (e - 4)) & 15) : (int)((d << (4 - e)) & 15);
    return (e << 4) | m;
}
constexpr int kBuckets = 64 * 16;

// per-block shared histogram, one global add per non-empty bucket (degrees
// crowd into a few buckets: same-address global atomics would serialise)
__global__ void deg_bucket_hist(int64_t n, const int64_t *__restrict__ rowptr, unsigned long long *bins) {
    __shared__ unsigned int h[kBuckets];
    for (int i = threadIdx.x; i < kBuckets; i += blockDim.x) h[i] = 0;
    __syncthreads();
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(h + deg_bucket(rowptr[v + 1] - rowptr[v]), 1u);
    __syncthreads();
    for (int i = threadIdx.x; i < kBuckets; i += blockDim.x)
        if (h[i]) atomicAdd(bins + i, (unsigned long long)h[i]);
}

// hub index of every vertex (-1: not a hub), by warp-aggregated appends:
// buckets >= btail take [0, KT) (cnt[0]), buckets in [brows, btail) take
// [KT, KR) (cnt[1] starts at KT), buckets in [bstar, brows) take [KR, K)
// (cnt[2] starts at KR); order inside each range is immaterial (keys carry
// the tie-break)
__global__ void hub_index_kernel(int64_t n, const int64_t *__restrict__ rowptr, int bstar, int brows, int btail,
                                 int32_t *hid, int32_t *hv, int32_t *cnt) {
    const int lane = threadIdx.x & 31;
    for (int64_t v0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) & ~31ll; v0 < n;
         v0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = v0 + lane;
        const int bk = v < n ? deg_bucket(rowptr[v + 1] - rowptr[v]) : -1;
        const int cls = bk >= btail ? 0 : (bk >= brows ? 1 : (bk >= bstar ? 2 : -1));
        int idx = -1;
#pragma unroll
        for (int c = 0; c < 3; ++c) {
            const unsigned m = __ballot_sync(0xffffffffu, cls == c);
            int b = 0;
            if (lane == 0 && m) b = atomicAdd(cnt + c, __popc(m));
            b = __shfl_sync(0xffffffffu, b, 0);
            if (cls == c) idx = b + __popc(m & lanemask_lt());
        }
        if (v < n) {
            hid[v] = idx;
            if (idx >= 0) hv[idx] = (int32_t)v;
        }
    }
}

// row h of M: warp per hub, the KW-word row gathered in shared memory
// (dynamic: 8 warps x KW words)
__global__ void __launch_bounds__(256) hub_matrix_kernel(int K, int KW, const int32_t *__restrict__ hv,
                                                         const int64_t *__restrict__ rowptr,
                                                         const int32_t *__restrict__ col,
                                                         const int32_t *__restrict__ hid,
                                                         const int32_t *__restrict__ thr, uint64_t *M,
                                                         unsigned long long *hkey) {
    extern __shared__ unsigned long long row_all[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    unsigned long long *row = row_all + (size_t)wid * KW;
    for (int h = blockIdx.x * 8 + wid; h < K; h += gridDim.x * 8) {
        for (int w = lane; w < KW; w += 32) row[w] = 0ull;
        __syncwarp();
        const int32_t v = hv[h];
        const int64_t eb = rowptr[v], ee = rowptr[v + 1];
        for (int64_t e0 = eb; e0 < ee; e0 += 128) {  // four independent gathers in flight per lane
            int32_t u[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) u[q] = e0 + 32 * q + lane < ee ? __ldg(col + e0 + 32 * q + lane) : -1;
#pragma unroll
            for (int q = 0; q < 4; ++q) u[q] = u[q] >= 0 ? __ldg(hid + u[q]) : -1;
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (u[q] >= 0) atomicOr(row + (u[q] >> 6), 1ull << (u[q] & 63));
        }
        __syncwarp();
        uint64_t *dst = M + (int64_t)h * KW;
        for (int w = lane; w < KW; w += 32) dst[w] = row[w];
        if (lane == 0) hkey[h] = pick_key(thr, v);
        __syncwarp();
    }
}

}  // namespace

HeuristicResult run_heuristic(mce_graph *g, int kind, int64_t h, int32_t shard_rank, int32_t shard_count,
                              bool want_runs, bool concurrent, bool with_core) {
    HeuristicResult res;
    const int64_t n = g->n;
    cudaStream_t s = concurrent ? g->hstream : g->stream;
    PinnedBuf &host = concurrent ? g->hhost : g->host;
    if (n == 0 || kind == 0) return res;
    bool use_core = (kind == 2 || kind == 4);
    bool single = (kind == 1 || kind == 2);
    if (single) h = 1;
    if (h <= 0 || h > n) h = n;
    if (use_core) {
        if (concurrent) fail(MCE_ERR_INVALID, "internal: core-number heuristics cannot overlap preprocessing");
        kcore(g);
    }
    cudaEvent_t e0, e1;
    MCE_CUDA(cudaEventCreate(&e0));
    MCE_CUDA(cudaEventCreate(&e1));
    MCE_CUDA(cudaEventRecord(e0, s));
    int64_t kernels = 0;

    Pool &pool = concurrent ? g->hpool : g->pool;
    pool.reset();
    const int32_t *thr;
    if (use_core) {
        thr = g->core.get();
    } else {
        int32_t *tb = pool.take<int32_t>(n);
        degree_thr_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), tb);
        MCE_LAUNCH_CHECK();
        ++kernels;
        thr = tb;
    }
    // ---- seeds: the h vertices with the highest threshold (ties: smaller id)
    int32_t *seeds = pool.take<int32_t>(n);
    int64_t nseeds = 0;
    if (h == n) {
        iota_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, seeds);
        MCE_LAUNCH_CHECK();
        ++kernels;
        nseeds = n;
    } else {
        int64_t maxthr = use_core ? g->degeneracy : g->max_deg;
        int64_t *bins = pool.take<int64_t>(maxthr + 1);
        MCE_CUDA(cudaMemsetAsync(bins, 0, sizeof(int64_t) * (maxthr + 1), s));
        thr_hist_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, thr, bins);
        MCE_LAUNCH_CHECK();
        int64_t *hb = host.get<int64_t>(maxthr + 1);
        MCE_CUDA(cudaMemcpyAsync(hb, bins, sizeof(int64_t) * (maxthr + 1), cudaMemcpyDeviceToHost, s));
        stream_sync(s);
        int64_t above = 0;
        int32_t tau = 0;
        for (int64_t t = maxthr; t >= 0; --t) {
            if (above + hb[t] >= h) {
                tau = (int32_t)t;
                break;
            }
            above += hb[t];
        }
        int64_t quota = h - above;
        int32_t *flag = pool.take<int32_t>(n);
        int64_t *pos = pool.take<int64_t>(n + 1), *tmp = pool.take<int64_t>(scan_tmp_items(n));
        tie_flags_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, thr, tau, flag);
        MCE_LAUNCH_CHECK();
        exclusive_scan_i32(flag, pos, n, tmp, s);
        seed_flags_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, thr, tau, pos, quota, flag);
        MCE_LAUNCH_CHECK();
        exclusive_scan_i32(flag, pos, n, tmp, s);
        compact_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, flag, pos, seeds);
        MCE_LAUNCH_CHECK();
        kernels += 10;
        nseeds = h;
    }
    // ---- shard the runs across ranks (cyclic over the id-ordered seed list)
    const int32_t *seed_ptr = seeds;
    if (shard_count > 1) {  // this rank's seeds: positions shard_rank, shard_rank + shard_count, ...
        const int64_t mine = nseeds > shard_rank ? (nseeds - shard_rank + shard_count - 1) / shard_count : 0;
        int32_t *sh = pool.take<int32_t>(std::max<int64_t>(mine, 1));
        if (mine > 0) {
            strided_gather_kernel<<<grid_for(mine, 256), 256, 0, s>>>(seeds + shard_rank, mine, shard_count, sh);
            MCE_LAUNCH_CHECK();
            ++kernels;
        }
        seed_ptr = sh;
        nseeds = mine;
    }
    // ---- the runs: hub seeds first (block per run), then the rest
    int32_t *scratch = pool.take<int32_t>(std::max<int64_t>(g->nnz, 1));
    int32_t *run_size = pool.take<int32_t>(n), *best = pool.take<int32_t>(1);
    unsigned long long *best_key = pool.take<unsigned long long>(1);
    int32_t *clique = pool.take<int32_t>(g->max_deg + 2);
    MCE_CUDA(cudaMemsetAsync(run_size, 0, sizeof(int32_t) * n, s));
    MCE_CUDA(cudaMemsetAsync(best, 0, sizeof(int32_t), s));
    MCE_CUDA(cudaMemsetAsync(best_key, 0, sizeof(unsigned long long), s));
    const int32_t *core = ((!concurrent || with_core) && g->have_core) ? g->core.get() : nullptr;
    const int abort_runs = want_runs ? 0 : 1;
    Hub H;
    int64_t nbig = 0;
    int32_t *big = nullptr;
    if (nseeds > 0 && g->max_deg > kBigSeed) {
        int32_t *flag = pool.take<int32_t>(nseeds);
        int64_t *pos = pool.take<int64_t>(nseeds + 1), *tmp = pool.take<int64_t>(scan_tmp_items(nseeds));
        big = pool.take<int32_t>(nseeds);
        big_flags_kernel<<<grid_for(nseeds, 256), 256, 0, s>>>(nseeds, seed_ptr, g->rowptr.get(), flag);
        MCE_LAUNCH_CHECK();
        exclusive_scan_i32(flag, pos, nseeds, tmp, s);
        gather_flagged_kernel<<<grid_for(nseeds, 256), 256, 0, s>>>(nseeds, seed_ptr, flag, pos, big);
        MCE_LAUNCH_CHECK();
        int64_t *hnb = host.get<int64_t>(1);
        MCE_CUDA(cudaMemcpyAsync(hnb, pos + nseeds, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        stream_sync(s);
        nbig = hnb[0];
        kernels += 5;
    }
    if (nbig >= 64) {  // enough hub runs for the hub bit matrix to pay
        // H = the vertices of the highest degree buckets: at most kHubBig of them
        // (and a matrix of at most a quarter of the free memory), the first
        // buckets up to kHubTail of them forming the tail set
        unsigned long long *bins = pool.take<unsigned long long>(kBuckets);
        MCE_CUDA(cudaMemsetAsync(bins, 0, sizeof(unsigned long long) * kBuckets, s));
        deg_bucket_hist<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), bins);
        MCE_LAUNCH_CHECK();
        unsigned long long *hb = host.get<unsigned long long>(kBuckets);
        MCE_CUDA(cudaMemcpyAsync(hb, bins, sizeof(unsigned long long) * kBuckets, cudaMemcpyDeviceToHost, s));
        stream_sync(s);
        const size_t free_b = dev_free_memory();
        unsigned long long kcap = kHubBig;
        while (kcap > kHubTail && (kcap * ((kcap + 63) / 64) * 8ull) > free_b / 4) kcap >>= 1;
        int bstar = kBuckets, btail = kBuckets, brows = kBuckets;
        unsigned long long above = 0, tail = 0, rows = 0;
        for (int b = kBuckets - 1; b >= 0; --b) {
            if (above + hb[b] > kcap) break;
            above += hb[b];
            if (hb[b]) bstar = b;
            if (above <= (unsigned long long)kHubTail) {
                tail = above;
                if (hb[b]) btail = b;
            }
            if (above <= (unsigned long long)kHubRows) {
                rows = above;
                if (hb[b]) brows = b;
            }
        }
        kernels += 1;
        if (above >= 64) {  // enough hubs to matter
            const int K = (int)above;
            const int KW = (K + 63) / 64;
            const int KR = std::max<int>((int)rows, (int)tail);
            int32_t *hid = pool.take<int32_t>(n), *hv = pool.take<int32_t>(K), *cnt = pool.take<int32_t>(3);
            const int32_t cnt0[3] = {0, (int32_t)tail, KR};
            MCE_CUDA(cudaMemcpyAsync(cnt, cnt0, sizeof(cnt0), cudaMemcpyHostToDevice, s));
            hub_index_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), bstar, brows, btail, hid, hv, cnt);
            MCE_LAUNCH_CHECK();
            // rows only for the KR highest-degree hubs (the picks of the runs; a
            // test against a lower pick falls back to the binary search), columns
            // for all K of them
            uint64_t *M = pool.take<uint64_t>((int64_t)KR * KW);
            unsigned long long *hkey = pool.take<unsigned long long>(K);
            const size_t smem = (size_t)8 * KW * sizeof(unsigned long long);
            MCE_CUDA(cudaFuncSetAttribute(hub_matrix_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            hub_matrix_kernel<<<std::max(1, std::min((KR + 7) / 8, num_sms() * 8)), 256, smem, s>>>(
                KR, KW, hv, g->rowptr.get(), g->col.get(), hid, thr, M, hkey);
            MCE_LAUNCH_CHECK();
            kernels += 2;
            H.hid = hid;
            H.hv = hv;
            H.hkey = hkey;
            H.M = M;
            H.K = K;
            H.KW = KW;
            H.KT = (int)tail;
            H.KR = KR;
        }
    }
    if (nseeds > 0) {
        if (nbig > 0) {
            // hub runs by descending degree, the first SM-count of them alone: the
            // longest runs publish their sizes before the rest start, which then abort
            // earlier (the order of runs never changes a result: ties go by key)
            int32_t *dk = pool.take<int32_t>(nbig), *dk2 = pool.take<int32_t>(nbig);
            int32_t *big2 = pool.take<int32_t>(nbig);
            seed_degree_kernel<<<grid_for(nbig, 256), 256, 0, s>>>(nbig, big, g->rowptr.get(), dk);
            MCE_LAUNCH_CHECK();
            size_t tb = 0;
            MCE_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, dk, dk2, big, big2, (int)nbig, 0, 32, s));
            void *tmpb = pool.take<uint8_t>((int64_t)tb);
            MCE_CUDA(cub::DeviceRadixSort::SortPairsDescending(tmpb, tb, dk, dk2, big, big2, (int)nbig, 0, 32, s));
            const int64_t first = std::min<int64_t>(nbig, num_sms());
            greedy_big_kernel<<<(int)first, kBlockRun, 0, s>>>(first, big2, g->rowptr.get(), g->col.get(), thr, core,
                                                               scratch, run_size, best, abort_runs, H);
            MCE_LAUNCH_CHECK();
            if (nbig > first) {
                const int blocks = (int)std::min<int64_t>(nbig - first, (int64_t)num_sms() * 4);
                greedy_big_kernel<<<blocks, kBlockRun, 0, s>>>(nbig - first, big2 + first, g->rowptr.get(),
                                                               g->col.get(), thr, core, scratch, run_size, best,
                                                               abort_runs, H);
                MCE_LAUNCH_CHECK();
            }
            kernels += 5;
        }
        greedy_kernel<<<grid_for(nseeds * 8, 256), 256, 0, s>>>(nseeds, seed_ptr, g->rowptr.get(), g->col.get(),
                                                                  thr, core, scratch, run_size, best, abort_runs, H);
        MCE_LAUNCH_CHECK();
        best_seed_kernel<<<grid_for(nseeds, 256), 256, 0, s>>>(nseeds, seed_ptr, thr, run_size, best, best_key);
        MCE_LAUNCH_CHECK();
        // (the winning run never picks a vertex of core + 1 < best: the same
        // filter leaves its picks unchanged, reading 15)
        replay_kernel<<<1, kReplay, 0, s>>>(best_key, best, abort_runs ? core : nullptr, g->rowptr.get(),
                                            g->col.get(), thr, scratch, clique, H);
        MCE_LAUNCH_CHECK();
        kernels += 3;
    }
    MCE_CUDA(cudaEventRecord(e1, s));
    int32_t *hbest = host.get<int32_t>(1);
    MCE_CUDA(cudaMemcpyAsync(hbest, best, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    stream_sync(s);
    res.omega_bar = hbest[0];
    float ms = 0;
    MCE_CUDA(cudaEventElapsedTime(&ms, e0, e1));
    res.ms = ms;
    res.kernels = kernels;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (res.omega_bar > 0) {
        res.clique.resize(res.omega_bar);
        MCE_CUDA(cudaMemcpyAsync(res.clique.data(), clique, sizeof(int32_t) * res.omega_bar, cudaMemcpyDeviceToHost,
                                 s));
        stream_sync(s);
    }
    if (want_runs) {
        res.run_size.resize(n);
        MCE_CUDA(cudaMemcpyAsync(res.run_size.data(), run_size, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, s));
        stream_sync(s);
    }
    return res;
}

}  // namespace mce
