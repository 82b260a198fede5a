// Frontier layout and expansion kernels (the hot path).
#pragma once

#include "graph.cuh"

namespace mce {

// One root of the current window.  Its candidate space is V = the root's
// out-neighbours (oriented CSR row, ranks ascending); local index i <-> V[L-1-i],
// i.e. bit order is REVERSE degeneracy order.  The colouring bound colours P
// in bit order and branches from the highest colour down (Tomita-Seki MCQ), so
// the high-core vertices get the low colours and are branched last, with the
// smallest candidate sets (the "smallest-last" initial order of Matula-Beck,
// DESIGN.md reading 5).  In ascending rank order the hub vertices took the
// highest colours and the R-MAT searches exploded.
struct RootInfo {
    int32_t r;      // rank of the root
    int32_t L;      // |V| = out-degree
    int64_t vbase;  // orp[r]: V = ocol + vbase
    int64_t abase;  // first word of the root's adjacency rows in the arena (L rows x W words)
};

// per-level arrays needed to read a clique back (PAPER.md IV-B: "sublistID ...
// allows us ... at the end of the computation, to read out all of the vertices")
struct LevelLink {
    const int32_t *parent;  // index of the parent entry in the previous level (-1 at level 1)
    const int32_t *vloc;    // local index of the vertex this entry added (-1 at level 1)
};

// A frontier level: |C| = k for every entry; P is the candidate set as a
// bitset over the root's local space (W words per entry, structure of arrays).
struct ExpandArgs {
    const uint64_t *P;
    const int32_t *slot;
    const int32_t *parent;
    const int32_t *vloc;
    int64_t begin, end;  // entries [begin, end) of the input level
    int32_t k;           // |C|
    int32_t need;        // smallest clique size still of interest
    int32_t bound;       // 0: |C|+|P|, 1: colouring
    int32_t Wp;          // words per candidate set of this level (kernel width; 1, 2, 4, 8, ...)
    int32_t Ps;          // P stride of this level in words (>= Wp: a fused pass writes the parent's width)
    int32_t Wa;          // words per adjacency row of the root window (>= Wp)
    int32_t Wc;          // write pass: words per child candidate set (<= Wp, from *maxbit)
    const RootInfo *roots;
    const uint64_t *adj;
    const int32_t *ocol;
    const int32_t *order;  // rank -> original vertex id
    // count pass
    int32_t *counts;  // indexed by entry
    // write pass
    const int64_t *offsets;  // exclusive scan of counts (indexed by entry)
    int64_t out_base;        // offsets[begin]
    uint64_t *cP;
    int32_t *cslot;
    int32_t *cparent;
    int32_t *cvloc;
    // count pass (atomicMax): maxbit[0] = highest candidate bit of any surviving
    // child, maxbit[1] = deepest level a descendant can reach (k + 1 + |P'|)
    int32_t *maxbit;
    // leaves of size k+1 (count pass only): total (exact) and staged rows
    unsigned long long *leaf_total;
    unsigned long long *leaf_slot;
    int32_t *leaf_rows;
    int64_t leaf_cap;  // rows
    const LevelLink *chain;  // chain[1..k]
    // clique completions (count pass, reading 10): an entry whose
    // candidate set P is itself a clique with k + |P| == need has exactly one
    // clique of interest below it, C + P; it is recorded (size need) instead of
    // expanded.  shortcut = 0 expands every level as Algorithm 2 does.
    int32_t shortcut;
    unsigned long long *clq_total;
    unsigned long long *clq_slot;
    int32_t *clq_rows;
    int64_t clq_cap;  // rows of `need` vertices
    // pair completions (reading 13): the count pass reserves their rows and
    // records (entry, first row, m) here; materialize_pairs writes the rows
    unsigned long long *pair_n;  // descriptors recorded
    int64_t *pair_desc;          // 3 x int64 each
    int64_t pair_cap;
    // fused count + write (count pass only): children are appended at
    // cP/cslot/... + atomicAdd(out_count) with stride Wp while they fit out_cap;
    // counts[] is written as usual so an overflowing level falls back to scan + write
    int32_t fused;
    unsigned long long *out_count;
    int64_t out_cap;
    // shared-memory path (expand_smem, count pass only): position q of the
    // level is entry perm[q] (entries grouped by root slot); blocks take
    // chunks of `chunk` positions from *chunk_ctr (zeroed by the caller)
    const int32_t *perm;
    unsigned long long *chunk_ctr;
    int32_t chunk;
    // re-rooted candidates (reroot_build_kernel): every root of this window is a
    // former candidate whose first k0 clique vertices (original ids) are
    // prefix[slot * k0 ..]; k0 = 0: ordinary roots (the clique starts at r)
    const int32_t *prefix;
    int32_t k0;
    // wide count pass (expand_wide, W >= 32): per-tile colouring-order scratch (u16 entries)
    uint16_t *wscratch;
    int64_t wscratch_n;
    long long *dbg;  // diagnostics (expand_small, verbose >= 2): cycles of the first entry's phases
    // universal-vertex rule (reading 19) in the thread path: the count and
    // write passes of one level must agree, so it is off when the level's count pass
    // is the shared-memory lockstep kernel (which does not apply it)
    int32_t universal;
};

// Fused root level for W == 1 roots (roots.cu): one warp per root builds the
// induced adjacency of V = N+(r), applies the bound and writes the level-2
// entries of surviving roots only.
struct RootArgs {
    const int32_t *list;  // roots: list[i * stride], i in [0, count)
    int64_t count, stride;
    const int64_t *orp;
    const int32_t *ocol;
    const int4 *ocol4;  // rows padded to 16-byte slots (mce_graph::ocol4) or nullptr
    const int32_t *order;
    int32_t need, bound;
    // outputs (appended; ctr = {roots, adjacency rows, level-2 entries, leaves})
    RootInfo *roots;
    uint64_t *adj;
    unsigned long long *ctr;
    uint64_t *cP;
    int32_t *cslot, *cparent, *cvloc;
    int32_t *leaf_rows;  // size-2 leaves (only when need <= 2)
    int64_t leaf_cap;
};
// max_len: an upper bound on |N+(r)| over the launch's roots (<= 4 selects the sparse kernel)
void launch_root_expand_w1(const RootArgs &a, int max_len, cudaStream_t s);

// Small-frontier fused levels (expand.cu expand_small): one block runs
// count -> scan -> write for consecutive levels while a level has at most
// kSmallMax entries of at most 4 words, so chains of tiny levels (the planted
// clique of er2000, the hub chain of R-MAT) cost one launch instead of ~7
// launches and a host round trip each.  It stops after a level that recorded
// leaves, produced more than kSmallMax children, or would not fit the scratch.
constexpr int kSmallMax = 1024;
constexpr int kSmallMaxLevels = 512;
struct SmallOut {
    int64_t status;    // 0: search below the input exhausted; 1: host continues with `children`;
                       // 2: stopped before processing level k_next (host processes it)
    int64_t levels;    // levels processed (|C| = k0 .. k0 + levels - 1)
    int64_t k_next;    // |C| of the level the host continues with
    int64_t children;  // its entries
    int64_t Wc;        // its word width
    int64_t Ps;        // its P stride in words (>= Wc)
    int64_t leaves;    // leaves (size k_next) recorded by the last processed level
    int64_t cliques;   // clique completions (size need) recorded by the last processed level
    uint64_t *P;       // the level the host continues with
    int32_t *slot, *parent, *vloc;
    uint64_t *inP;     // the last processed level (for a leaf replay)
    int32_t *inslot, *inparent, *invloc;
    int64_t inN, inW, inPs;
    int64_t level_n[kSmallMaxLevels];  // entries of every processed level
    long long prof[10];                // clock64 cycles per phase, summed over levels (verbose >= 2 prints them)
};
// write the rows of the pair completions recorded by the last count pass over
// the level described by `a` (its P / slot / chain); n = descriptors recorded
void launch_materialize_pairs(const ExpandArgs &a, int64_t n, cudaStream_t s);
void launch_expand_small(const ExpandArgs &a, uint8_t *scratch, int64_t scratch_bytes, SmallOut *out,
                         LevelLink *chain, cudaStream_t s);

// W classes: 0 -> 1 word, 1 -> 2, 2 -> 4, ... (W = 1 << class); L <= 64 W
constexpr int kMaxClass = 9;  // W up to 256 words (L <= 16384)

// bytes (optional): += the build's algorithmic bytes (build_adj_block, W >= 2)
void launch_build_adj(const RootInfo *roots, int64_t nroots, int W, const int64_t *orp, const int32_t *ocol,
                      uint64_t *adj, int64_t adj_words, cudaStream_t s, unsigned long long *bytes = nullptr);
void launch_init_level1(const RootInfo *roots, int64_t nroots, int W, uint64_t *P, int32_t *slot, int32_t *parent,
                        int32_t *vloc, cudaStream_t s);
void launch_expand(const ExpandArgs &a, bool write_pass, cudaStream_t s);
// widths the shared-memory count pass handles (the root's matrix, 64 W rows x W words, staged per block)
inline bool smem_width(int W) { return W == 4 || W == 8 || W == 16; }
// narrowest width the wide (global-row, lockstep) count pass takes: 32 words unless MCE_WIDE_MIN_W says otherwise
int wide_min_w();
// perm = the level's entries [0, n) grouped by slot (counting sort: hist over nslots, scan, scatter)
void launch_group_by_slot(const int32_t *slot, int64_t n, int32_t nslots, int32_t *hist, int64_t *offs,
                          int64_t *scan_tmp, int32_t *perm, cudaStream_t s);
// keep != nullptr: only CSR ids r >= keep_T with keep[r - keep_T] are roots (root colour filter, colour.cu)
void launch_classify_roots(int64_t n, const int64_t *orp, int32_t min_len, int32_t shard_rank, int32_t shard_count,
                           const uint8_t *keep, int64_t keep_T, int32_t *cls, int64_t *hist, cudaStream_t s);
// colour.cu: greedy colouring of the vertices of core >= need - 1 and the per-root colour bound
bool root_colour_filter(mce_graph *g, int32_t need, int64_t min_s, uint8_t *keep, int32_t *colr, int64_t *scratch,
                        cudaStream_t s, int64_t *T_out, int64_t *kept_out);
void launch_find_window(const int64_t *prefix, int64_t hi, int64_t lo_min, int64_t room, int64_t row_bytes,
                        int64_t per_root, int64_t *out, cudaStream_t s);
void launch_flag_eq(int64_t n, const int32_t *cls, int32_t c, int32_t *flag, cudaStream_t s);
void launch_compact(int64_t n, const int32_t *flag, const int64_t *pos, int32_t *out, cudaStream_t s);
void launch_make_roots(const int32_t *list, int64_t count, int64_t stride, int W, const int64_t *orp,
                       const int64_t *row_prefix, RootInfo *roots, cudaStream_t s);
void launch_root_lengths(const int32_t *list, int64_t count, int64_t stride, const int64_t *orp, int32_t *len,
                         cudaStream_t s);
// depth-d entry sharding (mce_options.shard_depth): flag[e] = 1 when the hash
// of entry e's vertex path (root CSR id, then the local vertices of levels
// 2..k) modulo `count` is `rank`; chain[2..k] must be set
// (a: roots, slot, chain, ocol, order, prefix / k0 of the level)
void launch_shard_flags(const ExpandArgs &a, int64_t n, int32_t k, int32_t rank, int32_t count, int32_t *flag,
                        cudaStream_t s);
// Re-rooting: each listed entry e of a level
// (candidate set P over its root's space of W words) becomes a root of its
// own whose space is P: L' = |P|, vertices V' (CSR ids, local index i <-> V'[L'-1-i],
// the old relative order kept), adjacency A' = the old rows of P's vertices
// compressed to P's bits (L' rows x Wn words), candidate set all of V', and a
// prefix of the entry's k clique vertices.  voff: exclusive scan of L' over the list.
void launch_reroot_sizes(const uint64_t *P, int Ps, int W, int64_t n, int32_t *Lp, int32_t *cls, int64_t *hist,
                         cudaStream_t s);
void launch_gather_i32(const int32_t *src, const int32_t *idx, int64_t n, int32_t *dst, cudaStream_t s);
void launch_reroot_build(const ExpandArgs &a, const int32_t *list, int64_t cnt, const int64_t *voff, int Wn,
                         int32_t *nV, uint64_t *nA, RootInfo *nroots, uint64_t *nP, int32_t *nslot, int32_t *nparent,
                         int32_t *nvloc, int32_t *nprefix, cudaStream_t s);
// out = the flagged entries of a level (P re-strided from Ps to W words)
void launch_gather_level(int64_t n, const int32_t *flag, const int64_t *pos, int W, int Ps, const uint64_t *P,
                         const int32_t *slot, const int32_t *parent, const int32_t *vloc, uint64_t *oP,
                         int32_t *oslot, int32_t *oparent, int32_t *ovloc, cudaStream_t s);
void launch_find_chunk_end(const int64_t *offsets, int64_t a, int64_t n, int64_t cap, int64_t *out,
                           cudaStream_t s);

}  // namespace mce
