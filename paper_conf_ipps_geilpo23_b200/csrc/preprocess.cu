// Preprocessing on the device (north star: "k-core/degeneracy ordering and
// edge orientation, done on device").
//
//  * kcore(): core numbers (PAPER.md II-B-2, line 61) by level peeling in ONE
//    cooperative persistent launch (kcore_async below): at level k every alive
//    vertex with degree <= k is appended to the peel order (core = k) and its
//    edges drained asynchronously, appending neighbours that fall to k.  The
//    peel order is a degeneracy order: when v is appended its remaining degree
//    (<= k) counts every neighbour appended after it, so orienting edges along
//    the order gives out-degree <= core(v) <= degeneracy.
//  * orient(): ranks (degeneracy = peel order, or degree order = PAPER.md IV-C
//    line 131 "keep the edge where the source vertex has lower degree") decide
//    the direction of every edge; the oriented CSR is stored in a second id
//    space ("CSR ids": vertices sorted by (core, degree) for the degeneracy
//    orientation, the rank itself for the degree orientation) with every row
//    sorted ascending.  The search colours candidates in reverse CSR-id order
//    (expand.cuh), i.e. high core first and, inside one core shell (where the
//    peel order is arbitrary), high degree first.
#include <cooperative_groups.h>

#include <cub/device/device_radix_sort.cuh>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "graph.cuh"

namespace cg = cooperative_groups;

namespace mce {

namespace {

constexpr int kPeelThreads = 1024;  // launch bound; the launch uses kcore_threads()

// ---------------------------------------------------------------------------
// k-core numbers and a degeneracy order: asynchronous level peel.  Within a level k the order in which
// queued vertices are processed does not matter: a vertex is appended to the
// peel order when its degree falls to <= k, and every neighbour appended after
// it was still unprocessed then, hence counted in that degree, so out-degrees
// along the order stay <= k (= its core number).  So a level runs as one
// asynchronous work list instead of one grid barrier per cascade round:
//
//   scan   : every alive vertex with degree <= k is appended (peel order,
//            core = k) and its edges are cut into work items of kChunk edges;
//            the rest is compacted into the next alive list
//   barrier
//   drain  : warps grab four work-list slots at a time (one atomicAdd), an
//            8-lane tile per item decrements the item's alive neighbours and
//            appends those that fall to k (tile-aggregated atomics); a slot
//            that is not yet written is polled until it is, or until every
//            reserved item is processed (done == tail: nothing can follow)
//   barrier, clear the level's work list, next level (k jumps to the
//            smallest alive degree when a scan appends nothing)
//
// Work items are int64 (vertex | chunk << 32), -1 = empty; levels alternate
// between two lists so one can be cleared while the other fills.
// ---------------------------------------------------------------------------
#ifndef ORIENT_KL
#define ORIENT_KL 4
#endif
#ifndef KCORE_OVL_PCT
#define KCORE_OVL_PCT 50  // percent of the SMs the peel takes beside the heuristic; measured 35 / 50 / 65 = ba1m 1.51 / 1.43 / 1.49 ms, rmat22 81.5 / 81.7 / 83.9 ms
#endif
#ifndef ORIENT_KL_DENSE
#define ORIENT_KL_DENSE 8  // (mean degree > 16) rmat22, round 2: 1 / 2 / 4 / 8 chunks = 37.8 / 36.8 / 36.6 / 36.2 ms per step
#endif
#ifndef KCORE_OVL_PCT_DENSE
#define KCORE_OVL_PCT_DENSE 30  // rmat22 after the round-2 heuristic work: 25 / 30 / 35 / 42% = 35.7 / 34.5 / 35.2 / 35.5 ms
#endif
#ifndef KCORE_CHUNK
#define KCORE_CHUNK 32  // measured: 128 / 64 / 32 / 16 / 8 = ba1m 1.49 / 1.46 / 1.43 / 1.44 / 1.50 ms, rmat22 82.5 / 81.8 / 82.1 / 81.4 / - ms
#endif
constexpr int64_t kChunk = KCORE_CHUNK;  // edges per work item
#ifndef KCORE_LOCAL
#define KCORE_LOCAL 0  // 1: fallen vertices continued by the same warp from a shared-memory stack (append_local); measured: rmat22 same, ba1m 1.40 -> 1.47-1.65 ms (20 ms without the batch cap: one warp serialises a long cascade)
#endif
#ifndef KCORE_LOCAL_BATCHES
#define KCORE_LOCAL_BATCHES 4
#endif
constexpr int kLocal = 96;  // items per warp-local continuation stack (32 warps x 768 B)
#ifndef KCORE_GRAB
#define KCORE_GRAB 0  // 1: reserve only while items are queued (fewer atomics on tiny levels); measured slower overall (rmat22 78.1 vs 74.2 ms, ba1m 1.52 vs 1.47)
#endif

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// append the vertices whose flag is set (tile of G lanes): peel order, core,
// dead, and ceil(deg / kChunk) work items each
template <int G>
__device__ __forceinline__ void async_append(bool take, int32_t u, const int64_t *__restrict__ rowptr, int32_t *core,
                                             int32_t *order, uint8_t *dead, long long *work,
                                             unsigned long long *otail, unsigned long long *wtail, int32_t k) {
    const int lane = threadIdx.x & 31;
    const int gl = lane & (G - 1), gbase = lane & ~(G - 1);
    const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
    const unsigned m = (__ballot_sync(gmask, take) & gmask) >> gbase;
    if (!m) return;
    int items = 0;
    if (take) {
        const int64_t d = rowptr[u + 1] - rowptr[u];
        items = (int)((d + kChunk - 1) / kChunk);
    }
    int inc = items;  // tile inclusive scan of item counts
#pragma unroll
    for (int o = 1; o < G; o <<= 1) {
        const int y = __shfl_up_sync(gmask, inc, o, G);
        if (gl >= o) inc += y;
    }
    const int total = __shfl_sync(gmask, inc, G - 1, G);
    unsigned long long ob = 0, wb = 0;
    if (gl == 0) {
        ob = atomicAdd(otail, (unsigned long long)__popc(m));
        if (total) wb = atomicAdd(wtail, (unsigned long long)total);
    }
    ob = __shfl_sync(gmask, ob, 0, G);
    wb = __shfl_sync(gmask, wb, 0, G);
    if (take) {
        order[ob + __popc(m & ((1u << gl) - 1u))] = u;
        core[u] = k;
        dead[u] = 1;
        for (int c = 0; c < items; ++c) work[wb + inc - items + c] = (long long)(uint32_t)u | ((long long)c << 32);
    }
}

// The drain's variant (whole warp): the vertices that fell are appended to
// the peel order as above, but their work items go to the warp's local stack
// (shared memory) while it has room -- the warp continues the cascade itself,
// depth first, instead of a round trip through the global list and another
// warp's poll (a cascade step then costs one warp's dependent loads).  Items
// that do not fit go to the global list.  lcount is warp-uniform.
__device__ __forceinline__ void append_local(bool take, int32_t u, const int64_t *__restrict__ rowptr, int32_t *core,
                                             int32_t *order, uint8_t *dead, long long *work,
                                             unsigned long long *otail, unsigned long long *wtail, int32_t k,
                                             long long *lstack, int &lcount, int lcap) {
    const int lane = threadIdx.x & 31;
    const unsigned m = __ballot_sync(0xffffffffu, take);
    if (!m) return;
    int items = 0;
    if (take) {
        const int64_t d = rowptr[u + 1] - rowptr[u];
        items = (int)((d + kChunk - 1) / kChunk);
    }
    int inc = items;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    const int total = __shfl_sync(0xffffffffu, inc, 31);
    const bool local = lcount + total <= lcap;
    unsigned long long ob = 0, wb = 0;
    if (lane == 0) {
        ob = atomicAdd(otail, (unsigned long long)__popc(m));
        if (total && !local) wb = atomicAdd(wtail, (unsigned long long)total);
    }
    ob = __shfl_sync(0xffffffffu, ob, 0);
    wb = __shfl_sync(0xffffffffu, wb, 0);
    if (take) {
        order[ob + __popc(m & lanemask_lt())] = u;
        core[u] = k;
        dead[u] = 1;
        for (int c = 0; c < items; ++c) {
            const long long it = (long long)(uint32_t)u | ((long long)c << 32);
            if (local)
                lstack[lcount + inc - items + c] = it;
            else
                work[wb + inc - items + c] = it;
        }
    }
    if (local) lcount += total;
    __syncwarp();
}

// ctrl (u64, one counter per 128-byte line so the hot counters do not share an
// L2 sector / slice): line 0 peel-order tail; lines 1..3 + 3 * (L % 2): work
// head, tail, done of level L; lines 8..11 + 4 * (s % 3): scan s appended /
// kept-alive count / min kept degree / dead entries seen
constexpr int kLine = 16;  // u64 per counter line
__global__ void __launch_bounds__(kPeelThreads)
    kcore_async(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col, int32_t *deg,
                int32_t *core, int32_t *order, int32_t *alive_a, int32_t *alive_b, uint8_t *dead,
                long long *work0, long long *work1, int64_t witems, unsigned long long *ctrl, int max_sleep,
                long long *trace) {
    cg::grid_group grid = cg::this_grid();
    __shared__ unsigned long long sh[8];
    __shared__ long long lstack_all[(kPeelThreads / 32) * kLocal];
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
    const int64_t nwarps = nthreads >> 5;
    const int lane = threadIdx.x & 31;
    unsigned long long *otail = ctrl;
#define CTR(i) (ctrl + kLine * (i))

    int64_t s = 0, L = 0;
    int64_t n_alive = n;
    int32_t *cur = alive_a, *nxt = alive_b;
    int32_t k = 0;
    bool compact = true;  // block-uniform: decided from counters every block reads after a grid barrier
    __shared__ unsigned swcnt[32];
    __shared__ unsigned long long sbase, sred[3][32];
    const int wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;
    while (true) {
        unsigned long long *head = CTR(1 + 3 * (L & 1)), *tail = CTR(2 + 3 * (L & 1)), *done = CTR(3 + 3 * (L & 1));
        unsigned long long *sapp = CTR(8 + 4 * (s % 3)), *skept = CTR(9 + 4 * (s % 3)), *smin = CTR(10 + 4 * (s % 3)),
                           *sdead = CTR(11 + 4 * (s % 3));
        long long *work = (L & 1) ? work1 : work0;
        if (tid == 0) {  // scan counters of s+1 (last read before scan s began)
            *CTR(8 + 4 * ((s + 1) % 3)) = 0;
            *CTR(9 + 4 * ((s + 1) % 3)) = 0;
            *CTR(10 + 4 * ((s + 1) % 3)) = ~0ull;
            *CTR(11 + 4 * ((s + 1) % 3)) = 0;
        }
        // ---- scan: append every alive vertex of degree <= k; the rest is
        // compacted into the next list only when enough of the list has died
        // (else the list is scanned in place next time, dead entries skipped).
        // Counts are aggregated per block (one atomic per block per scan, and
        // per block-iteration for the compaction offsets): same-address
        // atomics per warp cost ~n_alive / 32 serialised L2 operations per
        // scan, the larger part of a scan on rmat22 (260 scans, ~50 us each).
        int32_t dmin = INT32_MAX;
        unsigned napp = 0, ndead = 0;
        for (int64_t b0 = (int64_t)blockIdx.x * blockDim.x; b0 < n_alive; b0 += (int64_t)gridDim.x * blockDim.x) {
            const int64_t i = b0 + threadIdx.x;
            int32_t v = -1, d = 0;
            bool live = false;
            if (i < n_alive) {
                v = cur[i];
                live = !dead[v];
                if (live) d = deg[v];
                else ++ndead;
            }
            const bool q = live && d <= k;
            const bool keep = live && d > k;
            napp += q;
            async_append<32>(q, v, rowptr, core, order, dead, work, otail, tail, k);
            if (keep) dmin = min(dmin, d);
            if (compact) {
                const unsigned km = __ballot_sync(0xffffffffu, keep);
                if (lane == 0) swcnt[wib] = __popc(km);
                __syncthreads();
                if (wib == 0) {  // exclusive prefix over the block's warps, one atomic
                    const unsigned c = lane < nwb ? swcnt[lane] : 0u;
                    unsigned incl = c;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const unsigned y = __shfl_up_sync(0xffffffffu, incl, o);
                        if (lane >= o) incl += y;
                    }
                    if (lane < nwb) swcnt[lane] = incl - c;
                    const unsigned tot = __shfl_sync(0xffffffffu, incl, 31);
                    if (lane == 0) sbase = tot ? atomicAdd(skept, (unsigned long long)tot) : 0ull;
                }
                __syncthreads();
                if (keep) nxt[sbase + swcnt[wib] + __popc(km & lanemask_lt())] = v;
                __syncthreads();  // swcnt / sbase reuse
            }
        }
        {  // block totals: appended, dead entries seen, smallest kept degree
            const unsigned wa = __reduce_add_sync(0xffffffffu, napp), wd = __reduce_add_sync(0xffffffffu, ndead);
            const int32_t wm = __reduce_min_sync(0xffffffffu, dmin);
            if (lane == 0) {
                sred[0][wib] = wa;
                sred[1][wib] = wd;
                sred[2][wib] = (unsigned long long)(uint32_t)wm;
            }
            __syncthreads();
            if (wib == 0) {
                unsigned long long a = lane < nwb ? sred[0][lane] : 0ull, dd = lane < nwb ? sred[1][lane] : 0ull;
                unsigned long long m = lane < nwb ? sred[2][lane] : (unsigned long long)INT32_MAX;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    a += __shfl_xor_sync(0xffffffffu, a, o);
                    dd += __shfl_xor_sync(0xffffffffu, dd, o);
                    const unsigned long long y = __shfl_xor_sync(0xffffffffu, m, o);
                    m = y < m ? y : m;
                }
                if (lane == 0) {
                    if (a) atomicAdd(sapp, a);
                    if (dd) atomicAdd(sdead, dd);
                    if (m != (unsigned long long)INT32_MAX) atomicMin(smin, m);
                }
            }
        }
        grid.sync();
        if (threadIdx.x == 0) {
            sh[0] = __ldcg(sapp);
            sh[1] = __ldcg(skept);
            sh[2] = __ldcg(smin);
            sh[3] = __ldcg(otail);
            sh[4] = __ldcg(sdead);
        }
        __syncthreads();
        const unsigned long long appended = sh[0], kept = sh[1], md = sh[2], placed = sh[3], ndead_all = sh[4];
        __syncthreads();
        if (trace && tid == 0 && s < 8192) {  // MCE_KCORE_TRACE: (k, alive before scan, appended, t)
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            trace[8 * s] = k;
            trace[8 * s + 1] = n_alive;
            trace[8 * s + 2] = (long long)appended;
            trace[8 * s + 3] = (long long)t;
        }
        if (compact) {
            n_alive = (int64_t)kept;
            int32_t *t = cur;
            cur = nxt;
            nxt = t;
            compact = false;
        } else {
            compact = (ndead_all + appended) * 8 >= (unsigned long long)n_alive;
        }
        ++s;
        if ((int64_t)placed >= n) break;  // every vertex has its core number
        if (appended == 0) {              // nothing of degree <= k: jump to the smallest alive degree
            k = (int32_t)md;
            continue;
        }
        if (tid == 0) {  // counters of level L+1 (last read right after level L-1's drain)
            *CTR(1 + 3 * ((L + 1) & 1)) = 0;
            *CTR(2 + 3 * ((L + 1) & 1)) = 0;
            *CTR(3 + 3 * ((L + 1) & 1)) = 0;
        }
        // ---- drain the level's work list asynchronously.  A warp reserves four
        // slots (one per 8-lane tile) and polls them without blocking: an
        // unwritten slot may be waiting for an item that a sibling tile's item
        // appends.  The tiles' edge loops run in warp lock-step so appends and
        // done counts are aggregated over the whole warp (one atomic each).
        unsigned long long pending = 0;  // lane 0: items processed, not yet added to `done`
        bool finished = false;
        int next_rounds = 1;  // KCORE_GRAB == 2: rounds of 4 slots of the next reservation (lane 0)
        // warp-local continuation stack (append_local); pending is never
        // published while it holds items, so done < tail until it is empty
        long long *lst = lstack_all + (size_t)(threadIdx.x >> 5) * kLocal;
        int lcount = 0;
        // the edges of up to four items (one per 8-lane tile; -1: none), fallen
        // neighbours to the local stack
        auto run_items = [&](long long item) {
            int64_t eb = 0, ee = 0;
            if (item != -1) {
                const int32_t v = (int32_t)(item & 0xffffffffll);
                const int64_t c = item >> 32;
                eb = rowptr[v] + c * kChunk;
                ee = min(rowptr[v + 1], eb + kChunk);
            }
            const int iters = __reduce_max_sync(0xffffffffu, (unsigned)((ee - eb + 7) >> 3));
            for (int it = 0; it < iters; ++it) {
                const int64_t e = eb + it * 8 + (lane & 7);
                bool fell = false;
                int32_t u = -1;
                if (e < ee) {
                    u = col[e];
                    if (!dead[u]) fell = atomicSub(deg + u, 1) == k + 1;
                }
                if (KCORE_LOCAL)
                    append_local(fell, u, rowptr, core, order, dead, work, otail, tail, k, lst, lcount, kLocal);
                else
                    async_append<32>(fell, u, rowptr, core, order, dead, work, otail, tail, k);
            }
        };
        // pop up to four local items (one per tile) and run them, at most
        // KCORE_LOCAL_BATCHES times; what is left goes to the global list (a
        // long cascade must not serialise on one warp while others idle)
        auto drain_local = [&]() {
            int batches = 0;
            while (lcount > 0 && batches < KCORE_LOCAL_BATCHES) {
                const int take = min(lcount, 4);
                const int t = lane >> 3;
                const long long item = t < take ? lst[lcount - 1 - t] : -1ll;
                __syncwarp();
                lcount -= take;
                run_items(item);
                ++batches;
            }
            if (lcount > 0) {  // spill
                unsigned long long wb = 0;
                if (lane == 0) wb = atomicAdd(tail, (unsigned long long)lcount);
                wb = __shfl_sync(0xffffffffu, wb, 0);
                for (int i = lane; i < lcount; i += 32) work[wb + i] = lst[i];
                __syncwarp();
                lcount = 0;
            }
        };
        while (!finished) {
            // Lane 0 reserves slots only while the list holds unreserved items
            // (head < tail): with nothing queued, every warp reserving four
            // slots per level would cost one same-address atomic per warp
            // (~2400 per level, 959 levels on rmat22).  Otherwise it publishes
            // its processed count and waits until items arrive or done == tail
            // (read in that order: every appended item processed, nothing can
            // follow -- the level is over).  Deep backlogs are reserved in
            // groups of up to 8 rounds of 4 slots (fewer atomics on `head`).
            unsigned long long base = 0;
            int rounds = 0;
            if (lane == 0 && KCORE_GRAB == 2) {  // adaptive: grow while every slot was ready at once
                rounds = next_rounds;
                base = atomicAdd(head, 4ull * rounds);
            } else if (lane == 0 && !KCORE_GRAB) {
                base = atomicAdd(head, 4ull);
                rounds = 1;
            } else if (lane == 0) {
                int naps = 0;
                while (true) {
                    const unsigned long long h = ld_relaxed(head), t = ld_relaxed(tail);
                    if (h < t) {
                        const unsigned long long backlog = t - h;
                        rounds = backlog >= 64ull * (unsigned long long)nwarps ? 8 : (backlog >= 16ull * (unsigned long long)nwarps ? 2 : 1);
                        base = atomicAdd(head, 4ull * rounds);
                        break;
                    }
                    if (pending) {
                        __threadfence();  // this warp's appends before its done count
                        atomicAdd(done, pending);
                        pending = 0;
                    }
                    const unsigned long long dn = ld_relaxed(done), tl = ld_relaxed(tail);
                    if (dn == tl) break;  // rounds == 0: the level is over
                    __nanosleep(naps < 4 ? 32 : (naps < 16 ? 128 : max_sleep));
                    ++naps;
                }
            }
            base = __shfl_sync(0xffffffffu, base, 0);
            rounds = __shfl_sync(0xffffffffu, rounds, 0);
            if (rounds == 0) break;
          for (int rd = 0; rd < rounds && !finished; ++rd) {
            const unsigned long long slot = base + 4ull * rd + (lane >> 3);
            const int leader = lane & ~7;
            bool resolved = false, over = false;
            int idle = 0;  // consecutive empty polls: back off, and only then look at the hot counters
            int polls = 0;
            while (true) {
                long long item = -1;
                bool dead_slot = false;
                if (!resolved && (lane & 7) == 0) {
                    if (slot >= (unsigned long long)witems) {
                        dead_slot = true;  // beyond the list: can never be filled
                    } else {
                        item = (long long)ld_relaxed((const unsigned long long *)(work + slot));
                        if (item == -1 && idle >= 4) {
                            const unsigned long long dn = ld_relaxed(done);
                            const unsigned long long tl = ld_relaxed(tail);
                            dead_slot = dn == tl && slot >= tl;
                        }
                    }
                }
                item = __shfl_sync(0xffffffffu, item, leader);
                dead_slot = __shfl_sync(0xffffffffu, dead_slot, leader);
                const bool work_now = !resolved && item != -1;
                run_items(work_now ? item : -1ll);
                drain_local();  // the cascade below these items, in this warp
                const unsigned done_m = __ballot_sync(0xffffffffu, work_now && (lane & 7) == 0);
                if (lane == 0) pending += (unsigned long long)__popc(done_m);
                if (work_now) resolved = true;
                if (!resolved && dead_slot) {
                    resolved = true;
                    over = true;
                }
                ++polls;
                if (__all_sync(0xffffffffu, resolved)) break;
                if (!done_m) {
                    // about to wait: publish the processed count first (a warp with work
                    // batches it; termination needs every warp idle, hence flushed)
                    if (lane == 0 && pending) {
                        __threadfence();  // this warp's appends before its done count
                        atomicAdd(done, pending);
                        pending = 0;
                    }
                    ++idle;
                    __nanosleep(idle < 4 ? 32 : (idle < 16 ? 128 : max_sleep));
                } else {
                    idle = 0;
                }
            }
            if (__all_sync(0xffffffffu, over)) finished = true;  // later rounds' slots are beyond the end too
            if (KCORE_GRAB == 2 && lane == 0) next_rounds = polls == 1 ? min(8, next_rounds * 2) : 1;
          }
        }
        if (lane == 0 && pending) {  // (cannot happen: `over` needs an idle, flushed warp)
            __threadfence();
            atomicAdd(done, pending);
        }
        grid.sync();
        // ---- clear this level's work list (the next level fills the other one)
        if (threadIdx.x == 0) {
            sh[4] = __ldcg(head);
            sh[5] = __ldcg(tail);
        }
        __syncthreads();
        const int64_t extent = min((int64_t)max(sh[4], sh[5]), witems);
        const int64_t placed2 = (int64_t)__ldcg(otail);
        __syncthreads();
        if (trace && tid == 0 && s - 1 < 8192) {  // drain end, items drained, vertices placed
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            trace[8 * (s - 1) + 4] = (long long)t;
            trace[8 * (s - 1) + 5] = (long long)sh[5];
            trace[8 * (s - 1) + 6] = placed2;
        }
        for (int64_t i = tid; i < extent; i += nthreads) work[i] = -1;
        ++L;
        ++k;
        if (placed2 >= n) break;
    }
}
#undef CTR

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

// sort key of the CSR id space: core * (max_deg + 1) + degree
__global__ void priority_keys_kernel(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ core,
                                     uint64_t span, uint64_t *keys, int32_t *vals) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        keys[v] = (core ? (uint64_t)(uint32_t)core[v] * span : 0ull) + (uint64_t)(rowptr[v + 1] - rowptr[v]);
        vals[v] = (int32_t)v;
    }
}

__global__ void invert_kernel(int64_t n, const int32_t *__restrict__ order, int32_t *rank) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        rank[order[i]] = (int32_t)i;
}

// Tile of G lanes (4, 8 or 32) inside a warp: lane index, first lane, member mask.
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

// count + stage: the up-neighbours of v (as CSR ids) are written compacted at
// the start of v's own undirected row in `stage` (rowptr-indexed), their
// number at odeg[pid[v]]; orient_copy moves them to the oriented CSR once the
// out-degrees are scanned (one gather pass over rank/pid instead of two)
// (rank, CSR id) of a vertex in one 8-byte word: the stage pass gathers both
// with one load per neighbour (one sector instead of two)
__global__ void pack_rank_pid_kernel(int64_t n, const int32_t *__restrict__ rank, const int32_t *__restrict__ pid,
                                     int2 *rp) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        rp[v] = make_int2(rank[v], pid[v]);
}

template <int G, int KL>
__device__ void stage_one(int64_t v, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                          const int2 *__restrict__ rp, int32_t *odeg, int32_t *stage) {
    Tile<G> t;
    const int2 rv = rp[v];
    const int32_t r = rv.x;
    const int64_t eb = rowptr[v], ee = rowptr[v + 1];
    int64_t out = eb;
    // KL chunks' ids and ranks gathered before any is used, so a row costs
    // one gather latency per KL chunks
    constexpr int K = KL;
    for (int64_t e0 = eb; e0 < ee; e0 += G * K) {
        int32_t u[K];
        int2 x[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const int64_t e = e0 + G * k + t.gl;
            u[k] = e < ee ? col[e] : -1;
        }
#pragma unroll
        for (int k = 0; k < K; ++k) x[k] = u[k] >= 0 ? __ldg(rp + u[k]) : make_int2(INT32_MIN, 0);
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const bool up = x[k].x > r;
            const unsigned m = t.ballot(up);
            if (up) stage[out + __popc(m & t.lt())] = x[k].y;
            out += __popc(m);
        }
    }
    if (t.gl == 0) odeg[rv.y] = (int32_t)(out - eb);
}

// Warp w takes vertices [Vw, Vw+V), V = 32 / TG: TG-lane tiles (TK chunks
// per trip) when all V have degree <= 64, else a warp each (KL chunks per
// trip).  Measured (`profiles/r02_orient_tile_ab_v1.txt`): 8-lane tiles for
// sparse graphs (ba1m preprocessing 1.08 ms vs 1.12 with 4-lane tiles),
// 4-lane tiles with 2 chunks per trip for mean degree > 16 (rmat22 18.0 ->
// 17.75 ms).
template <int KL, int TG, int TK>
__global__ void __launch_bounds__(256) orient_stage_kernel(int64_t n, const int64_t *__restrict__ rowptr,
                                                           const int32_t *__restrict__ col,
                                                           const int2 *__restrict__ rp, int32_t *odeg,
                                                           int32_t *stage) {
    constexpr int V = 32 / TG;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t v0 = warp * V; v0 < n; v0 += nwarps * V) {
        const int64_t v = v0 + lane / TG;
        const int64_t d = v < n ? rowptr[v + 1] - rowptr[v] : 0;
        if (__all_sync(0xffffffffu, d <= 64)) {
            if (v < n) stage_one<TG, TK>(v, rowptr, col, rp, odeg, stage);
        } else {
            for (int t = 0; t < V && v0 + t < n; ++t) stage_one<32, KL>(v0 + t, rowptr, col, rp, odeg, stage);
        }
        __syncwarp();
    }
}

// oriented row of CSR id i = the staged prefix of vertex vid[i]'s row (8-lane
// tile per row, 4 rows per warp; a warp per row when a row exceeds 64)
__global__ void __launch_bounds__(256) orient_copy_kernel(int64_t n, const int64_t *__restrict__ rowptr,
                                                          const int32_t *__restrict__ vid,
                                                          const int64_t *__restrict__ orp,
                                                          const int32_t *__restrict__ stage, int32_t *ocol) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t i0 = warp * 4; i0 < n; i0 += nwarps * 4) {
        const int64_t i = i0 + (lane >> 3);
        int64_t ob = 0, len = 0, sb = 0;
        if (i < n) {
            ob = orp[i];
            len = orp[i + 1] - ob;
            sb = rowptr[vid[i]];
        }
        if (__all_sync(0xffffffffu, len <= 64)) {
            for (int64_t j = lane & 7; j < len; j += 8) ocol[ob + j] = stage[sb + j];
        } else {
            for (int t = 0; t < 4; ++t) {
                const int64_t bo = __shfl_sync(0xffffffffu, ob, 8 * t), bl = __shfl_sync(0xffffffffu, len, 8 * t);
                const int64_t bs = __shfl_sync(0xffffffffu, sb, 8 * t);
                for (int64_t j = lane; j < bl; j += 32) ocol[bo + j] = stage[bs + j];
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
// rows by length class: (32, 256] -> mid and (256, 1024] -> wide (a warp each,
// in registers), (1024, 8192] -> big (a block each, shared memory), longer ->
// huge (one block, global scratch); meta = counts [mid, big, huge], the largest
// out-degree, count [wide]
__global__ void long_rows_kernel(int64_t n, const int64_t *__restrict__ orp, int32_t *mid, int32_t *big,
                                 int32_t *huge, int32_t *wide, int32_t *meta) {
    const int lane = threadIdx.x & 31;
    int32_t mx = 0;
    for (int64_t r0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) & ~31ll; r0 < n;
         r0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = r0 + lane;
        const int32_t len = r < n ? (int32_t)(orp[r + 1] - orp[r]) : 0;
        mx = max(mx, len);
        const int cls = len <= 32 ? -1 : (len <= 256 ? 0 : (len <= 1024 ? 3 : (len <= 8192 ? 1 : 2)));
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            const unsigned m = __ballot_sync(0xffffffffu, cls == c);
            int32_t b = 0;
            if (lane == 0 && m) b = atomicAdd(meta + (c == 3 ? 4 : c), __popc(m));
            b = __shfl_sync(0xffffffffu, b, 0);
            int32_t *dst = c == 0 ? mid : (c == 1 ? big : (c == 2 ? huge : wide));
            if (cls == c) dst[b + __popc(m & lanemask_lt())] = (int32_t)r;
        }
    }
    mx = __reduce_max_sync(0xffffffffu, mx);
    if (lane == 0 && mx) atomicMax(meta + 3, mx);
}

// rows of (32, 32 E] ids by one warp each, E per lane in registers ("blocked":
// lane l holds positions l E .. l E + E - 1): a bitonic network whose strides
// below E stay inside a lane and the rest are lane shuffles -- no barrier
// (a 256-thread block per row with a barrier per stage was 3.3 ms on rmat22)
template <int E>
__global__ void __launch_bounds__(256) sort_rows_mid(const int64_t *__restrict__ orp, int32_t *ocol,
                                                      const int32_t *__restrict__ rows, int32_t nrows) {
    const int lane = threadIdx.x & 31;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t ri = warp; ri < nrows; ri += nwarps) {
        const int32_t r = rows[ri];
        const int64_t b = orp[r];
        const int len = (int)(orp[r + 1] - b);
        int32_t x[E];
#pragma unroll
        for (int j = 0; j < E; ++j) {
            const int i = lane * E + j;
            x[j] = i < len ? ocol[b + i] : INT32_MAX;
        }
#pragma unroll
        for (int size = 2; size <= 32 * E; size <<= 1) {
#pragma unroll
            for (int stride = size >> 1; stride > 0; stride >>= 1) {
                if (stride >= E) {
#pragma unroll
                    for (int j = 0; j < E; ++j) {
                        const int i = lane * E + j;
                        const int32_t y = __shfl_xor_sync(0xffffffffu, x[j], stride / E);
                        const bool up = (i & size) == 0, lower = (i & stride) == 0;
                        x[j] = (lower == up) ? min(x[j], y) : max(x[j], y);
                    }
                } else {
#pragma unroll
                    for (int j = 0; j < E; ++j) {
                        const int p = j ^ stride;
                        if (p > j) {
                            const bool up = ((lane * E + j) & size) == 0;
                            const int32_t a = x[j], c = x[p];
                            x[j] = up ? min(a, c) : max(a, c);
                            x[p] = up ? max(a, c) : min(a, c);
                        }
                    }
                }
            }
        }
#pragma unroll
        for (int j = 0; j < E; ++j) {
            const int i = lane * E + j;
            if (i < len) ocol[b + i] = x[j];
        }
    }
}

// ---------------------------------------------------------------------------
// Deterministic degeneracy order (MCE_ORIENT_DEGENERACY_DET, multi-GPU): the
// asynchronous peel above gives every vertex its (unique) core number but a
// peel ORDER that depends on timing, and root / candidate sharding needs every
// rank to orient the edges identically.  With the core numbers known, shell c
// (the vertices of core c) is peeled inside the c-core H_c in synchronous
// rounds, every shell at once:
//   d(v)  = neighbours w with core(w) >= core(v)        (degree inside H_c)
//   round t removes every alive v with d(v) <= core(v) (a set fixed by the
//           state at the start of the round), then decrements d(w) for the
//           alive neighbours w of the same shell
// Each round's set, hence round(v), is a function of the graph alone.  Order
// = (core, round, id): when v goes (round t) every later neighbour -- higher
// core, or same shell with round >= t -- was alive and counted in d(v) <=
// core(v), so out-degrees along the order stay <= core (a degeneracy order).
// One cooperative launch, two grid barriers per round; frontier lists
// alternate.  ctrl[0] = rounds, ctrl[2 + (t & 1)] = size of frontier t.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(512)
    shell_round_peel(int64_t n, const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                     const int32_t *__restrict__ core, int32_t *d, int32_t *round, int32_t *fa, int32_t *fb,
                     unsigned long long *ctrl) {
    cg::grid_group grid = cg::this_grid();
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
    const int lane = threadIdx.x & 31;
    // d(v) and frontier 0: a warp per 32 vertices, 8-lane tiles over the rows
    // (rows of more than 64 neighbours by the whole warp: a hub's row is
    // 4x shorter per lane)
    for (int64_t v0 = (tid >> 5) * 32; v0 < n; v0 += (nthreads >> 5) * 32) {
        for (int q = 0; q < 32; q += 4) {
            const int64_t v = v0 + q + (lane >> 3);
            int32_t cnt = 0, c = 0;
            int64_t eb = 0, ee = 0;
            if (v < n) {
                c = core[v];
                eb = rowptr[v];
                ee = rowptr[v + 1];
            }
            const bool longrow = ee - eb > 64;
            if (v < n && !longrow)
                for (int64_t e = eb + (lane & 7); e < ee; e += 8) cnt += core[col[e]] >= c;
            cnt += __shfl_xor_sync(0xffffffffu, cnt, 1);
            cnt += __shfl_xor_sync(0xffffffffu, cnt, 2);
            cnt += __shfl_xor_sync(0xffffffffu, cnt, 4);
            const unsigned lm = __ballot_sync(0xffffffffu, longrow && (lane & 7) == 0);
            for (unsigned mm = lm; mm; mm &= mm - 1) {  // the tiles' long rows, one at a time by the warp
                const int src = __ffs(mm) - 1;
                const int64_t lb = __shfl_sync(0xffffffffu, eb, src), le = __shfl_sync(0xffffffffu, ee, src);
                const int32_t lc = __shfl_sync(0xffffffffu, c, src);
                int32_t lcnt = 0;
                for (int64_t e = lb + lane; e < le; e += 32) lcnt += core[col[e]] >= lc;
                lcnt = __reduce_add_sync(0xffffffffu, lcnt);
                if (lane == src) cnt = lcnt;
            }
            const bool take = v < n && (lane & 7) == 0 && cnt <= c;
            if (v < n && (lane & 7) == 0) {
                d[v] = cnt;
                round[v] = -1;
            }
            const unsigned m = __ballot_sync(0xffffffffu, take);
            unsigned long long b = 0;
            if (lane == 0 && m) b = atomicAdd(ctrl + 2, (unsigned long long)__popc(m));
            b = __shfl_sync(0xffffffffu, b, 0);
            if (take) fa[b + __popc(m & lanemask_lt())] = (int32_t)v;
        }
    }
    grid.sync();
    int32_t *cur = fa, *nxt = fb;
    for (int32_t t = 0;; ++t) {
        const int64_t nf = (int64_t)__ldcg(ctrl + 2 + (t & 1));
        if (nf == 0) {
            if (tid == 0) ctrl[0] = (unsigned long long)t;
            break;
        }
        for (int64_t i = tid; i < nf; i += nthreads) round[cur[i]] = t;
        if (tid == 0) ctrl[2 + ((t + 1) & 1)] = 0;
        grid.sync();
        // decrements: 8-lane tile per frontier vertex
        for (int64_t b0 = (tid >> 5) * 4; b0 < nf; b0 += (nthreads >> 5) * 4) {  // warp-uniform trip count
            const int64_t i = b0 + (lane >> 3);
            int32_t v = -1, c = 0;
            int64_t eb = 0, ee = 0;
            if (i < nf) {
                v = cur[i];
                c = core[v];
                eb = rowptr[v];
                ee = rowptr[v + 1];
            }
            // rows of more than 64 neighbours by the whole warp, the rest by 8-lane tiles
            const bool longrow = ee - eb > 64;
            const unsigned lm = __ballot_sync(0xffffffffu, longrow && (lane & 7) == 0);
            const int64_t seb = longrow ? 0 : eb, see = longrow ? 0 : ee;
            const int iters = __reduce_max_sync(0xffffffffu, (unsigned)((see - seb + 7) >> 3));
            for (int it = 0; it < iters; ++it) {
                const int64_t e = seb + it * 8 + (lane & 7);
                bool fell = false;
                int32_t w = -1;
                if (e < see) {
                    w = col[e];
                    if (core[w] == c && __ldcg(round + w) < 0) fell = atomicSub(d + w, 1) == c + 1;
                }
                const unsigned m = __ballot_sync(0xffffffffu, fell);
                unsigned long long b = 0;
                if (lane == 0 && m) b = atomicAdd(ctrl + 2 + ((t + 1) & 1), (unsigned long long)__popc(m));
                b = __shfl_sync(0xffffffffu, b, 0);
                if (fell) nxt[b + __popc(m & lanemask_lt())] = w;
            }
            for (unsigned mm = lm; mm; mm &= mm - 1) {
                const int src = __ffs(mm) - 1;
                const int64_t lb = __shfl_sync(0xffffffffu, eb, src), le = __shfl_sync(0xffffffffu, ee, src);
                const int32_t lc = __shfl_sync(0xffffffffu, c, src);
                for (int64_t e0 = lb; e0 < le; e0 += 32) {
                    const int64_t e = e0 + lane;
                    bool fell = false;
                    int32_t w = -1;
                    if (e < le) {
                        w = col[e];
                        if (core[w] == lc && __ldcg(round + w) < 0) fell = atomicSub(d + w, 1) == lc + 1;
                    }
                    const unsigned m = __ballot_sync(0xffffffffu, fell);
                    unsigned long long b = 0;
                    if (lane == 0 && m) b = atomicAdd(ctrl + 2 + ((t + 1) & 1), (unsigned long long)__popc(m));
                    b = __shfl_sync(0xffffffffu, b, 0);
                    if (fell) nxt[b + __popc(m & lanemask_lt())] = w;
                }
            }
        }
        grid.sync();
        int32_t *tmp = cur;
        cur = nxt;
        nxt = tmp;
    }
}

// sort key of the deterministic order: core * (rounds + 1) + round (stable radix sort: ties by id)
__global__ void shell_keys_kernel(int64_t n, const int32_t *__restrict__ core, const int32_t *__restrict__ round,
                                  uint64_t span, uint64_t *keys, int32_t *vals) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        keys[v] = (uint64_t)(uint32_t)core[v] * span + (uint64_t)(uint32_t)round[v];
        vals[v] = (int32_t)v;
    }
}

// stable radix sort of `keys` (values: vertex ids ascending) into `out`
void sort_by_key_stable(uint64_t *keys, uint64_t *keys_out, int32_t *vals, int32_t *out, int64_t n, uint64_t kmax,
                        mce::Pool &pool, cudaStream_t s) {
    int end_bit = 1;
    while (end_bit < 64 && (1ull << end_bit) <= kmax) ++end_bit;
    size_t tmp_bytes = 0;
    MCE_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, keys, keys_out, vals, out, (int)n, 0, end_bit, s));
    void *tmp = pool.take<uint8_t>((int64_t)tmp_bytes);
    MCE_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, keys, keys_out, vals, out, (int)n, 0, end_bit, s));
}

// g->order = the deterministic degeneracy order (needs g->core)
void deterministic_order(mce_graph *g) {
    const int64_t n = g->n;
    cudaStream_t s = g->stream;
    int32_t *d = g->pool.take<int32_t>(n), *round = g->pool.take<int32_t>(n);
    int32_t *fa = g->pool.take<int32_t>(n), *fb = g->pool.take<int32_t>(n);
    unsigned long long *ctrl = g->pool.take<unsigned long long>(4);
    MCE_CUDA(cudaMemsetAsync(ctrl, 0, 4 * sizeof(unsigned long long), s));
    int blocks_per_sm = 0;
    MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, shell_round_peel, 512, 0));
    if (blocks_per_sm < 1) fail(2, "shell_round_peel: cooperative kernel does not fit an SM");
    // (all SMs even beside the heuristic: the rounds are the longer branch --
    // rmat22 with the k-core's 30% share 57.9 ms per step, with all SMs 54.4)
    const int grid = num_sms() * std::min(blocks_per_sm, 2);
    int64_t n_arg = n;
    const int64_t *rp = g->rowptr.get();
    const int32_t *cl = g->col.get(), *co = g->core.get();
    unsigned long long *ct = ctrl;
    void *args[] = {&n_arg, &rp, &cl, &co, &d, &round, &fa, &fb, &ct};
    MCE_CUDA(cudaLaunchCooperativeKernel((void *)shell_round_peel, grid, 512, args, 0, s));
    unsigned long long *h = g->host.get<unsigned long long>(1);
    MCE_CUDA(cudaMemcpyAsync(h, ctrl, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    stream_sync(s);
    const uint64_t span = h[0] + 1;
    uint64_t *keys = g->pool.take<uint64_t>(n), *keys_out = g->pool.take<uint64_t>(n);
    int32_t *vals = g->pool.take<int32_t>(n);
    shell_keys_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->core.get(), round, span, keys, vals);
    MCE_LAUNCH_CHECK();
    sort_by_key_stable(keys, keys_out, vals, g->order.get(), n, ((uint64_t)g->degeneracy + 1) * span, g->pool, s);
    g->kernels += 4;
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
    // work items: at most one per vertex plus one per kChunk edges, per level list
    const int64_t witems = n + g->nnz / kChunk + 1;
    long long *work0 = g->pool.take<long long>(witems), *work1 = g->pool.take<long long>(witems);
    unsigned long long *ctrl = g->pool.take<unsigned long long>(kLine * 20);
    MCE_CUDA(cudaMemsetAsync(dead, 0, n, s));
    MCE_CUDA(cudaMemsetAsync(work0, 0xff, sizeof(long long) * witems, s));
    MCE_CUDA(cudaMemsetAsync(work1, 0xff, sizeof(long long) * witems, s));
    MCE_CUDA(cudaMemsetAsync(ctrl, 0, kLine * 20 * sizeof(unsigned long long), s));
    for (int i = 0; i < 3; ++i)  // smin of the three scan counter sets
        MCE_CUDA(cudaMemsetAsync(ctrl + kLine * (10 + 4 * i), 0xff, sizeof(unsigned long long), s));
    degrees_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), deg, alive_a);
    MCE_LAUNCH_CHECK();
    // launch shape (measured on B200, ba1m / rmat22): alone, one 512-thread
    // block per SM; overlapped with the heuristic (engine.cu), 1024-thread
    // blocks on half of the SMs, leaving the other half to the heuristic
    // (ba1m 1.88 -> 1.74 ms, rmat22 221 -> 190 ms per step).  Fewer, wider
    // blocks contend less on the work-list counters.
    const bool half = g->pre_overlapped;
    const int threads = half ? 1024 : 512;
    int blocks_per_sm = 0;
    MCE_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, kcore_async, threads, 0));
    if (blocks_per_sm < 1) fail(2, "kcore: cooperative kernel does not fit an SM");
    // beside the heuristic: a smaller share on graphs of mean degree > 16, whose
    // heuristic is long and whose peel gains nothing from more blocks (rmat22:
    // 20 / 27 / 35 / 42 / 50% = 40.4 / 38.3 / 37.7 / 38.1 / 39.0 ms per step,
    // re-swept after the later heuristic changes: 30% best; ba1m keeps 50%:
    // 35% = 1.45 ms, 42% = 1.37, 50% = 1.37)
    const int pct = g->nnz > 16 * n ? KCORE_OVL_PCT_DENSE : KCORE_OVL_PCT;
    const int grid = half ? std::max(1, num_sms() * pct / 100) : num_sms();
    int64_t n_arg = n;
    const int64_t *rp = g->rowptr.get();
    const int32_t *cl = g->col.get();
    int32_t *dg = deg, *co = g->core.get(), *qu = g->peel.get(), *aa = alive_a, *ab = alive_b;
    uint8_t *dd = dead;
    long long *w0 = work0, *w1 = work1;
    int64_t wi = witems;
    unsigned long long *ct = ctrl;
    int ms = 512;  // longest poll back-off (ns); 256-2048 measured equal
    long long *trace = nullptr;
    const bool tracing = getenv("MCE_KCORE_TRACE") != nullptr;  // per-scan trace to stderr (tuning aid)
    if (tracing) {
        trace = g->pool.take<long long>(8 * 8192);
        MCE_CUDA(cudaMemsetAsync(trace, 0xff, sizeof(long long) * 8 * 8192, s));
    }
    void *args[] = {&n_arg, &rp, &cl, &dg, &co, &qu, &aa, &ab, &dd, &w0, &w1, &wi, &ct, &ms, &trace};
    MCE_CUDA(cudaLaunchCooperativeKernel((void *)kcore_async, grid, threads, args, 0, s));
    if (tracing) {
        std::vector<long long> ht(8 * 8192);
        MCE_CUDA(cudaMemcpyAsync(ht.data(), trace, sizeof(long long) * ht.size(), cudaMemcpyDeviceToHost, s));
        stream_sync(s);
        fprintf(stderr, "[kcore] grid %d x %d\n", grid, threads);
        for (int i = 0; i < 8192 && ht[8 * i] >= 0; ++i)
            fprintf(stderr, "[kcore] scan %d k %lld alive %lld appended %lld t_us %.2f drain_end_us %.2f items %lld placed %lld\n",
                    i, ht[8 * i], ht[8 * i + 1], ht[8 * i + 2], (ht[8 * i + 3] - ht[3]) / 1e3,
                    ht[8 * i + 4] >= 0 ? (ht[8 * i + 4] - ht[3]) / 1e3 : -1.0, ht[8 * i + 5], ht[8 * i + 6]);
    }
    g->kernels += 2;
    // degeneracy = max core (the last queued vertex has it)
    last_core_kernel<<<1, 1, 0, s>>>(n, g->peel.get(), g->core.get(), deg);
    int32_t *h = g->host.get<int32_t>(1);
    MCE_CUDA(cudaMemcpyAsync(h, deg, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    stream_sync(s);
    g->degeneracy = h[0];
    g->have_core = true;
}

// Out-rows of <= 4 ids padded to one aligned 16-byte slot per vertex (-1
// fill): the sparse root level (roots.cu root_expand_l4) then fetches a row
// with one LDG.128 and no row bounds -- two dependent loads per root instead
// of four.
__global__ void pad_rows4_kernel(int64_t n, const int64_t *__restrict__ orp, const int32_t *__restrict__ ocol,
                                 int4 *__restrict__ out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = orp[v];
        const int d = (int)(orp[v + 1] - b);
        int4 x;
        x.x = d > 0 ? ocol[b] : -1;
        x.y = d > 1 ? ocol[b + 1] : -1;
        x.z = d > 2 ? ocol[b + 2] : -1;
        x.w = d > 3 ? ocol[b + 3] : -1;
        out[v] = x;
    }
}

#ifndef PAD_ROWS4
#define PAD_ROWS4 1
#endif
void orient(mce_graph *g, int orientation) {
    if (g->orientation == orientation) return;
    g->have_ocol4 = false;
    const int64_t n = g->n;
    cudaStream_t s = g->stream;
    g->order.ensure(std::max<int64_t>(n, 1));
    g->rank.ensure(std::max<int64_t>(n, 1));
    g->vid.ensure(std::max<int64_t>(n, 1));
    g->pid.ensure(std::max<int64_t>(n, 1));
    g->orp.ensure(n + 1);
    g->ocol.ensure(std::max<int64_t>(g->nnz / 2, 1) + 4);  // + 4: int4 over-reads of the root level (roots.cu load4)
    g->pool.reset();
    if (n == 0) {
        MCE_CUDA(cudaMemsetAsync(g->orp.get(), 0, sizeof(int64_t), s));
        g->orientation = orientation;
        g->max_out = 0;
        return;
    }
    if (g->order_given) {  // mce_set_order: g->order already holds the order
    } else if (orientation == 0) {  // degeneracy: the peel queue
        MCE_CUDA(cudaMemcpyAsync(g->order.get(), g->peel.get(), sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
    } else if (orientation == 2) {  // deterministic degeneracy order: (core, shell round, id)
        deterministic_order(g);
    } else {  // degree order, ties by vertex id (a stable radix sort: deterministic, so every rank
              // of a sharded run orients identically)
        uint64_t *keys = g->pool.take<uint64_t>(n), *keys_out = g->pool.take<uint64_t>(n);
        int32_t *vals = g->pool.take<int32_t>(n);
        priority_keys_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), nullptr, 0, keys, vals);
        MCE_LAUNCH_CHECK();
        sort_by_key_stable(keys, keys_out, vals, g->order.get(), n, (uint64_t)g->max_deg + 1, g->pool, s);
        g->kernels += 4;
    }
    invert_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->order.get(), g->rank.get());
    MCE_LAUNCH_CHECK();
    // id space of the oriented CSR (reading 5): degeneracy -> vertices
    // sorted by (core, degree) ascending, so the reverse local order of a root
    // meets high-core, then high-degree vertices first; degree -> the rank itself
    if (orientation != 1) {
        uint64_t *keys = g->pool.take<uint64_t>(n), *keys_out = g->pool.take<uint64_t>(n);
        int32_t *vals = g->pool.take<int32_t>(n);
        const uint64_t span = (uint64_t)g->max_deg + 1;
        priority_keys_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rowptr.get(), g->core.get(), span, keys, vals);
        MCE_LAUNCH_CHECK();
        // only as many radix bits as the largest key needs (BA 1M: 15 bits, 2 passes)
        const uint64_t kmax = ((uint64_t)g->degeneracy + 1) * span;
        int end_bit = 1;
        while (end_bit < 64 && (1ull << end_bit) < kmax) ++end_bit;
        size_t tmp_bytes = 0;
        MCE_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, keys, keys_out, vals, g->vid.get(), (int)n, 0,
                                                 end_bit, s));
        void *tmp = g->pool.take<uint8_t>((int64_t)tmp_bytes);
        MCE_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, keys, keys_out, vals, g->vid.get(), (int)n, 0,
                                                 end_bit, s));
        invert_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->vid.get(), g->pid.get());
        MCE_LAUNCH_CHECK();
        g->kernels += 4;
    } else {
        MCE_CUDA(cudaMemcpyAsync(g->vid.get(), g->order.get(), sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
        MCE_CUDA(cudaMemcpyAsync(g->pid.get(), g->rank.get(), sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
    }
    int32_t *odeg = g->pool.take<int32_t>(n);
    int32_t *stage = g->pool.take<int32_t>(std::max<int64_t>(g->nnz, 1));
    // Long rows (degree > 64, a warp each) gather ORIENT_KL chunks per trip when
    // they are rare (mean degree <= 16: ba1m preprocessing 1.27 -> 1.17 ms) and
    // ORIENT_KL_DENSE otherwise (round 1, beside a 44 ms heuristic, 4 chunks
    // slowed rmat22's step 82.6 -> 88-93 ms; round 2, beside a 20 ms one, they
    // gain 37.8 -> 36.6 ms)
    int2 *rp2 = g->pool.take<int2>(n);
    pack_rank_pid_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->rank.get(), g->pid.get(), rp2);
    MCE_LAUNCH_CHECK();
    if (g->nnz <= 16 * n)
        orient_stage_kernel<ORIENT_KL, 8, 1><<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->rowptr.get(), g->col.get(), rp2,
                                                                                 odeg, stage);
    else
        orient_stage_kernel<ORIENT_KL_DENSE, 4, 2><<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->rowptr.get(), g->col.get(),
                                                                                       rp2, odeg, stage);
    MCE_LAUNCH_CHECK();
    exclusive_scan_i32(odeg, g->orp.get(), n, g->pool.take<int64_t>(scan_tmp_items(n)), s);
    orient_copy_kernel<<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->rowptr.get(), g->vid.get(), g->orp.get(), stage,
                                                             g->ocol.get());
    MCE_LAUNCH_CHECK();
    sort_rows_warp<<<grid_for(n * 8, 256), 256, 0, s>>>(n, g->orp.get(), g->ocol.get());
    MCE_LAUNCH_CHECK();
    int32_t *rmid = g->pool.take<int32_t>(n), *rbig = g->pool.take<int32_t>(n), *rhuge = g->pool.take<int32_t>(n);
    int32_t *rwide = g->pool.take<int32_t>(n);
    int32_t *meta = g->pool.take<int32_t>(5);
    MCE_CUDA(cudaMemsetAsync(meta, 0, 5 * sizeof(int32_t), s));
    long_rows_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->orp.get(), rmid, rbig, rhuge, rwide, meta);
    MCE_LAUNCH_CHECK();
    int32_t *hmeta = g->host.get<int32_t>(5);
    MCE_CUDA(cudaMemcpyAsync(hmeta, meta, 5 * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    stream_sync(s);
    g->kernels += 8;
    g->max_out = hmeta[3];
    g->have_ocol4 = false;
    if (g->max_out <= 4 && PAD_ROWS4) {  // (rows this short need no further sort)
        g->ocol4.ensure(n);
        pad_rows4_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->orp.get(), g->ocol.get(), g->ocol4.get());
        MCE_LAUNCH_CHECK();
        g->kernels += 1;
        g->have_ocol4 = true;
    }
    const int32_t n_mid = hmeta[0], n_big = hmeta[1], n_huge = hmeta[2], n_wide = hmeta[4];
    const int32_t smem_cap = 8192;  // ints (32 KB)
    if (n_mid > 0) {
        sort_rows_mid<8><<<grid_for((int64_t)n_mid * 32, 256), 256, 0, s>>>(g->orp.get(), g->ocol.get(), rmid, n_mid);
        MCE_LAUNCH_CHECK();
        g->kernels += 1;
    }
    if (n_wide > 0) {
        sort_rows_mid<32><<<grid_for((int64_t)n_wide * 32, 256), 256, 0, s>>>(g->orp.get(), g->ocol.get(), rwide,
                                                                               n_wide);
        MCE_LAUNCH_CHECK();
        g->kernels += 1;
    }
    if (n_big > 0) {
        sort_rows_block<<<grid_for(n_big, 1, 16), 256, smem_cap * sizeof(int32_t), s>>>(
            g->orp.get(), g->ocol.get(), rbig, n_big, nullptr, smem_cap);
        MCE_LAUNCH_CHECK();
        g->kernels += 1;
    }
    if (n_huge > 0) {  // rows beyond shared memory: one block, global scratch
        int32_t p2 = 1;
        while (p2 < g->max_out) p2 <<= 1;
        int32_t *scratch = g->pool.take<int32_t>(p2);
        sort_rows_block<<<1, 1024, smem_cap * sizeof(int32_t), s>>>(g->orp.get(), g->ocol.get(), rhuge, n_huge,
                                                                    scratch, smem_cap);
        MCE_LAUNCH_CHECK();
        g->kernels += 1;
    }
    g->orientation = orientation;  // (stream-ordered: no sync needed before the consumers)
}

void orient_from(mce_graph *g, int orientation, const int32_t *order, bool on_device) {
    kcore(g);  // core numbers (deterministic) for the CSR-id space and the heuristics
    const int64_t n = g->n;
    g->order.ensure(std::max<int64_t>(n, 1));
    if (n)
        MCE_CUDA(cudaMemcpyAsync(g->order.get(), order, sizeof(int32_t) * n,
                                 on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, g->stream));
    g->order_given = true;
    g->orientation = -1;
    orient(g, orientation);
    g->order_given = false;
    stream_sync(g->stream);
}

__global__ void max_core_kernel(int64_t n, const int32_t *__restrict__ core, int32_t *out) {
    int m = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        m = max(m, core[v]);
    for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0) atomicMax(out, m);
}

// Multi-GPU: rank 0 peels once, the others take its
// core numbers and peel order instead of re-peeling -- the asynchronous peel's
// order depends on timing, and root / candidate ownership needs every rank to
// orient the edges the same way.  The degeneracy is max core (recomputed, so a
// degree-ordered `peel` would still give the right value).
void set_core(mce_graph *g, const int32_t *core, const int32_t *peel, bool on_device) {
    const int64_t n = g->n;
    cudaStream_t s = g->stream;
    g->core.ensure(std::max<int64_t>(n, 1));
    g->peel.ensure(std::max<int64_t>(n, 1));
    g->have_core = false;
    g->orientation = -1;  // the oriented CSR (and its CSR-id priorities) follow the new cores
    g->degeneracy = 0;
    if (n) {
        const auto kind = on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
        MCE_CUDA(cudaMemcpyAsync(g->core.get(), core, sizeof(int32_t) * n, kind, s));
        MCE_CUDA(cudaMemcpyAsync(g->peel.get(), peel, sizeof(int32_t) * n, kind, s));
        g->pool.reset();
        int32_t *mx = g->pool.take<int32_t>(1);
        MCE_CUDA(cudaMemsetAsync(mx, 0, sizeof(int32_t), s));
        max_core_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, g->core.get(), mx);
        MCE_LAUNCH_CHECK();
        int32_t *h = g->host.get<int32_t>(1);
        MCE_CUDA(cudaMemcpyAsync(h, mx, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
        stream_sync(s);
        g->degeneracy = h[0];
    }
    g->have_core = true;
}

bool preprocessed(const mce_graph *g, int orientation) {
    return g->orientation == orientation && (g->have_core || orientation == 1);
}

void preprocess(mce_graph *g, int orientation) {
    if (preprocessed(g, orientation)) return;
    if (!g->pre_ev[0]) {
        MCE_CUDA(cudaEventCreate(&g->pre_ev[0]));
        MCE_CUDA(cudaEventCreate(&g->pre_ev[1]));
    }
    if (!g->pre_started) MCE_CUDA(cudaEventRecord(g->pre_ev[0], g->stream));  // (else the caller's, before its kcore)
    g->pre_started = false;
    g->kernels = 0;
    // the degree orientation (PAPER.md IV-C) needs no core numbers: the k-core
    // peel runs only for the degeneracy orientations (and on demand for the
    // core-number heuristics, mce_preprocess and the root colour filter)
    if (orientation != 1) kcore(g);
    orient(g, orientation);
    // no host sync here: the device time is read after the caller's next one
    MCE_CUDA(cudaEventRecord(g->pre_ev[1], g->stream));
    g->pre_pending = true;
}

double preprocess_ms(mce_graph *g) {
    if (g->pre_pending) {
        MCE_CUDA(cudaEventSynchronize(g->pre_ev[1]));
        float ms = 0;
        MCE_CUDA(cudaEventElapsedTime(&ms, g->pre_ev[0], g->pre_ev[1]));
        g->t_pre_ms = ms;
        g->pre_pending = false;
    }
    return g->t_pre_ms;
}

}  // namespace mce
