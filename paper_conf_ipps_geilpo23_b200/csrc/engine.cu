// Breadth-first maximum clique driver (PAPER.md IV-D Algorithm 2 MAXCLIQUES,
// IV-E windowed search) over the device kernels of expand.cu.
//
//  run():   preprocess -> heuristic lower bound -> roots grouped by candidate
//           set width W -> windows of roots -> level-synchronous expansion.
//  process(k): one level: count pass (+ leaf capture) -> scan -> write pass
//           of the next level -> recurse.  When the next level would exceed
//           the frontier budget it is produced and explored in chunks
//           (the paper's windowing applied at any depth, V-C-3 "Recursive
//           Windowing"), so the frontier never exceeds the budget.
#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <exception>
#include <thread>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <vector>

#include "engine.cuh"
#include "expand.cuh"
#include "canon.cuh"
#include "heuristic.cuh"

namespace mce {

namespace {
constexpr size_t kAlign = 256;

// Bump allocator over the graph's workspace segments, limited to the budget.
// Segments are allocated on demand (the first sized for a typical run, later
// ones kBigSeg or larger) and kept on the graph handle for the next call, so
// small problems stay small while an exploding frontier may use the whole
// budget.  Allocation is stack-like: mark() / reset(mark).
constexpr size_t kBigSeg = 4ull << 30;
#ifndef PRE_PRIORITY
#define PRE_PRIORITY 0  // 1: preprocessing beside the heuristic on a greatest-priority stream (measured: no change, rmat22 43.2 vs 43.1 ms)
#endif
#ifndef KCORE_FIRST
#define KCORE_FIRST 0  // 1: the peel alone first, then the heuristic (with core numbers) beside the orientation; measured slower (rmat22 54.6 vs 46.7 ms, ba1m 1.80 vs 1.38)
#endif
constexpr int64_t kLevelReserve = 12 * (int64_t)kAlign;  // see process(): chunk sizing (the fixed allocations of one level)
// the root colour filter runs when at least this many vertices can be in a
// clique of the size sought (below it the colouring costs more than it saves;
// MCE_ROOT_COLOUR_MIN_S overrides, for tests)
constexpr int64_t kRootColourMinS = 4096;
struct Arena {
    struct Mark {
        size_t seg, off, before;
    };
    std::vector<DevBuf<uint8_t>> *segs = nullptr;
    size_t budget = 0, first = 0;
    size_t cur = 0, off = 0, before = 0;  // before = bytes of the segments below cur
    void init(std::vector<DevBuf<uint8_t>> &s, size_t budget_bytes, size_t first_seg) {
        segs = &s;
        budget = budget_bytes;
        first = std::min(first_seg, budget_bytes);
        cur = off = before = 0;
        if (segs->empty() || (*segs)[0].n < first) {
            segs->clear();
            segs->emplace_back();
            (*segs)[0].alloc(first);
        }
    }
    size_t used() const { return before + off; }
    size_t avail() const { return budget > used() ? budget - used() : 0; }
    Mark mark() const { return {cur, off, before}; }
    void reset(const Mark &m) {
        cur = m.seg;
        off = m.off;
        before = m.before;
    }
    // at != nullptr: receives the mark just before the allocation (after a segment switch)
    template <typename T>
    T *alloc(int64_t count, Mark *at = nullptr) {
        const size_t bytes = ((size_t)std::max<int64_t>(count, 1) * sizeof(T) + kAlign - 1) / kAlign * kAlign;
        if (off + bytes > (*segs)[cur].n) {  // next segment (the rest of this one is skipped)
            const size_t nb = before + (*segs)[cur].n;
            if (nb + bytes > budget)
                fail(MCE_ERR_BUDGET, "frontier budget exhausted (need " + std::to_string(bytes) + " more bytes, " +
                                         std::to_string(avail()) + " available)");
            const size_t want = std::min(std::max(kBigSeg, bytes), budget - nb);
            if (cur + 1 >= segs->size()) segs->emplace_back();
            if ((*segs)[cur + 1].n < bytes) (*segs)[cur + 1].alloc(want);
            before = nb;
            ++cur;
            off = 0;
        }
        if (used() + bytes > budget)
            fail(MCE_ERR_BUDGET, "frontier budget exhausted (need " + std::to_string(bytes) + " more bytes, " +
                                     std::to_string(avail()) + " available)");
        T *p = reinterpret_cast<T *>((*segs)[cur].p + off);
        if (at) *at = Mark{cur, off, before};
        off += bytes;
        return p;
    }
};

struct Level {
    int64_t count = 0;
    int32_t W = 1;   // words per candidate set (kernel width)
    int32_t Ps = 0;  // P stride in words (0: = W; a fused pass writes the parent's width)
    uint64_t *P = nullptr;
    int32_t *slot = nullptr;
    int32_t *parent = nullptr;
    int32_t *vloc = nullptr;
};

class Timer {
   public:
    explicit Timer(cudaStream_t s) : s_(s) {
        MCE_CUDA(cudaEventCreate(&a_));
        MCE_CUDA(cudaEventCreate(&b_));
    }
    ~Timer() {
        cudaEventDestroy(a_);
        cudaEventDestroy(b_);
    }
    void start() { MCE_CUDA(cudaEventRecord(a_, s_)); }
    void stop() { MCE_CUDA(cudaEventRecord(b_, s_)); pending_ = true; }
    // accumulate after the stream has been synchronised past stop()
    double collect() {
        if (!pending_) return 0.0;
        float ms = 0;
        MCE_CUDA(cudaEventElapsedTime(&ms, a_, b_));
        pending_ = false;
        return ms;
    }

   private:
    cudaStream_t s_;
    cudaEvent_t a_, b_;
    bool pending_ = false;
};

// Per-launch device timing of the expansion kernels without a host sync per
// launch: event pairs are recorded around each launch and read once the
// stream has been synchronised (collect()), then reused.
class LaunchClock {
   public:
    explicit LaunchClock(cudaStream_t s) : s_(s) {}
    ~LaunchClock() {
        for (auto &e : ev_) {
            cudaEventDestroy(e.a);
            cudaEventDestroy(e.b);
        }
    }
    // kind: 0 count pass, 1 write pass, 2 fused root level, 3 root setup (root
    // colour filter, re-root matrix builds), 4 root matrix builds (build_adj_block);
    // 3 and 4 are not part of the expansion total
    int start(int kind) {
        if (used_ == ev_.size()) {
            Pair p;
            MCE_CUDA(cudaEventCreate(&p.a));
            MCE_CUDA(cudaEventCreate(&p.b));
            ev_.push_back(p);
        }
        ev_[used_].kind = kind;
        MCE_CUDA(cudaEventRecord(ev_[used_].a, s_));
        return (int)used_++;
    }
    void stop(int i) { MCE_CUDA(cudaEventRecord(ev_[i].b, s_)); }
    // call after a stream sync that covers every recorded pair
    void collect(double &all_ms, double &count_ms, double &root_ms, double &setup_ms, double &build_ms) {
        for (size_t i = 0; i < used_; ++i) {
            float ms = 0;
            MCE_CUDA(cudaEventElapsedTime(&ms, ev_[i].a, ev_[i].b));
            if (ev_[i].kind >= 3) {
                setup_ms += ms;
                if (ev_[i].kind == 4) build_ms += ms;
                continue;
            }
            all_ms += ms;
            if (ev_[i].kind == 0) count_ms += ms;
            if (ev_[i].kind == 2) root_ms += ms;
        }
        used_ = 0;
    }

   private:
    struct Pair {
        cudaEvent_t a, b;
        int kind;
    };
    cudaStream_t s_;
    std::vector<Pair> ev_;
    size_t used_ = 0;
};

// verbose > 1: device time of one step, synchronously (diagnostics only)
template <typename F>
double timed_step(cudaStream_t s, bool on, F &&f) {
    if (!on) {
        f();
        return 0.0;
    }
    cudaEvent_t a, b;
    MCE_CUDA(cudaEventCreate(&a));
    MCE_CUDA(cudaEventCreate(&b));
    MCE_CUDA(cudaEventRecord(a, s));
    f();
    MCE_CUDA(cudaEventRecord(b, s));
    MCE_CUDA(cudaEventSynchronize(b));
    float ms = 0;
    MCE_CUDA(cudaEventElapsedTime(&ms, a, b));
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    return ms;
}

class Engine {
   public:
    Engine(mce_graph *g, const mce_options &o, bool find_one)
        : g_(g), o_(o), find_one_(find_one), s_(g->stream), clock_(g->stream) {}

    mce_result *run();

   private:
    int32_t need() const { return find_one_ ? best_ + 1 : best_; }
    void process(int32_t k, const Level &L);
    bool run_small(int32_t k, const Level &L);
    bool reroot(int32_t k, const Level &L);
    void do_class(int32_t cls, const int32_t *list, int64_t count);
    void do_class_w1(const int32_t *list, int64_t count);
    void handle_leaves(int32_t size, int64_t cnt, ExpandArgs &a, int kind = 0);
    void leaf_args(ExpandArgs &a) const;
    void materialize_pairs(ExpandArgs &a);
    void reset_leaf_counters() {
        MCE_CUDA(cudaMemsetAsync(leaf_total_, 0, 4 * sizeof(unsigned long long), s_));
        MCE_CUDA(cudaMemsetAsync(pair_n_, 0, sizeof(unsigned long long), s_));
    }
    void sync_bound(bool active);
    void launch_timed(const ExpandArgs &a, bool write);

    mce_graph *g_;
    mce_options o_;
    bool find_one_;
    cudaStream_t s_;
    LaunchClock clock_;
    Arena arena_;
    int32_t best_ = 0;
    int32_t W_ = 1;   // words per adjacency row of the current root window
    int64_t stride_ = 1, offset_ = 0;
    bool entry_shard_ = false;  // shard_depth >= 2: levels < depth replicated, level-depth entries dealt by hash
    bool split_ = false;        // inside a subtree whose level-depth entries were dealt

    // leaves
    unsigned long long *leaf_total_ = nullptr;  // g->misc[0]
    unsigned long long *leaf_slot_ = nullptr;   // g->misc[1]
    unsigned long long *clq_total_ = nullptr;   // g->misc[2] clique completions (reading 10)
    unsigned long long *clq_slot_ = nullptr;    // g->misc[3]
    int32_t *maxbit_ = nullptr;                 // g->misc[4]
    unsigned long long *out_count_ = nullptr;   // g->misc[5] fused-pass children
    unsigned long long *build_bytes_ = nullptr; // g->misc[8] algorithmic bytes of the root matrix builds
    int64_t build_launches_ = 0;
    unsigned long long *pair_n_ = nullptr;      // g->misc[6] pair-completion descriptors
    unsigned long long *chunk_ctr_ = nullptr;   // g->misc[7] work counter of the shared-memory count pass
    int64_t nroots_ = 0;                        // roots of the current window (slots 0 .. nroots_ - 1)
    const int32_t *vtab_ = nullptr;             // vertex table of the window's roots (g->ocol, or re-rooted lists)
    const int32_t *prefix_ = nullptr;           // re-rooted window: per-root clique prefix (k0_ vertices each)
    int32_t k0_ = 0;
    // levels this wide re-root their candidates (0: never, the default: on rmat26
    // the re-root matrix builds cost 17.5 s for no expansion gain -- 48.7 s vs
    // 30.2 s per step, 40.8 s with 64; MCE_REROOT_MIN_W sets it, tests force it)
    int reroot_min_w_ = 0;
    int32_t no_reroot_level_ = -1;              // the level being processed in a re-rooted space
    int smem_min_w_ = 8;                        // narrowest level width taking the shared-memory count pass
    int64_t smem_min_n_ = 2048;                 // ... and fewest entries (small levels: rows stay L1/L2 hits)
    int64_t smem_per_root_ = 16;                // ... and fewest entries per root of the window on average
    int64_t pair_cap_ = 0;
    int64_t stage_rows_ = 0;
    int64_t cstage_rows_ = 0;
    int64_t stage_max_rows_ = 0;  // staging never exceeds a quarter of the budget (stored list truncated, count exact)
    std::vector<int32_t> rows_;  // find-one: the clique held on the host (width res_size_)
    int64_t stored_ = 0;         // enumerate: rows kept in g->store (device, width res_size_)
    int32_t res_size_ = 0;
    int64_t res_count_ = 0;
    bool truncated_ = false;

    // chain of levels for clique read-out (device copy in g->misc)
    LevelLink *chain_dev_ = nullptr;
    int32_t chain_cap_ = 0;

    const RootInfo *roots_ = nullptr;
    const uint64_t *adj_ = nullptr;

    // stats
    std::vector<int64_t> level_entries_;
    double t_expand_ms_ = 0.0, t_count_ms_ = 0.0, t_root_ms_ = 0.0, t_setup_ms_ = 0.0, t_build_ms_ = 0.0;
    int64_t count_launches_ = 0, kernels_ = 0, root_launches_ = 0;
    double count_bytes_ = 0.0, root_bytes_ = 0.0;
};

void Engine::launch_timed(const ExpandArgs &a, bool write) {
    const int t = clock_.start(write ? 1 : 0);
    launch_expand(a, write, s_);
    clock_.stop(t);
    ++kernels_;
    if (!write) {
        ++count_launches_;
        const double n = (double)(a.end - a.begin);
        count_bytes_ += n * (8.0 * a.Wp + 4 + 4 + 4 + sizeof(RootInfo));
    }
}

void Engine::sync_bound(bool active) {
    if (!o_.bound_sync) return;
    int32_t gactive = 0;
    int32_t gb = o_.bound_sync(best_, active ? 1 : 0, &gactive, o_.bound_sync_user);
    if (gb < 0) fail(MCE_ERR_SYNC, "bound_sync reported a failed exchange");
    if (gb > best_) best_ = gb;
}

void Engine::leaf_args(ExpandArgs &a) const {
    a.leaf_total = leaf_total_;
    a.leaf_slot = leaf_slot_;
    a.leaf_rows = g_->stage.get();
    a.leaf_cap = stage_rows_;
    // No clique / pair completions above the split depth of the level-d deal:
    // whether a completion fires depends on this shard's bound (k + |P| ==
    // need), so a clique could be completed above the split on one shard and
    // reached below it on another.  Without them, what is found above the split
    // (leaves only) does not depend on the bound, and every deeper clique sits
    // under exactly one dealt level-d entry.
    a.shortcut = (o_.no_clique_shortcut || (entry_shard_ && !split_)) ? 0 : 1;
    a.universal = 1;  // (process() turns it off for levels counted by the lockstep kernel)
    a.clq_total = clq_total_;
    a.clq_slot = clq_slot_;
    a.clq_rows = g_->cstage.get();
    a.clq_cap = cstage_rows_;
    a.pair_n = pair_n_;
    a.pair_desc = g_->pdesc.get();
    a.pair_cap = pair_cap_;
}

// Pair completions (reading 13): the count pass reserved their staging rows
// and left descriptors; write the rows (growing the descriptor list and
// replaying the count pass once if it overflowed)
void Engine::materialize_pairs(ExpandArgs &a) {
    for (int attempt = 0; attempt < 2; ++attempt) {
        unsigned long long *hp = g_->host.get<unsigned long long>(1);
        MCE_CUDA(cudaMemcpyAsync(hp, pair_n_, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        const int64_t np = (int64_t)hp[0];
        if (np > a.pair_cap && attempt == 0) {
            pair_cap_ = np;
            g_->pdesc.ensure((size_t)pair_cap_ * 3);
            a.pair_desc = g_->pdesc.get();
            a.pair_cap = pair_cap_;
            reset_leaf_counters();
            launch_expand(a, false, s_);
            ++kernels_;
            continue;
        }
        launch_materialize_pairs(a, std::min<int64_t>(np, a.pair_cap), s_);
        ++kernels_;
        return;
    }
}

// Record `cnt` cliques of `size` staged by a count pass: kind 0 = leaves
// C + {v} (a.leaf_rows), kind 1 = clique completions C + P (a.clq_rows).
void Engine::handle_leaves(int32_t size, int64_t cnt, ExpandArgs &a, int kind) {
    if (cnt <= 0) return;
    if (entry_shard_ && !split_ && offset_ != 0) {  // found above the split depth by every shard: shard 0 reports
        if (size > best_) best_ = size;
        return;
    }
    DevBuf<int32_t> &stage = kind ? g_->cstage : g_->stage;
    if (kind == 1) materialize_pairs(a);
    if (find_one_) {
        // all cliques of this launch have size > best: keep the first
        best_ = size;
        res_size_ = size;
        res_count_ = 1;
        rows_.resize(size);
        MCE_CUDA(cudaMemcpyAsync(rows_.data(), stage.get(), sizeof(int32_t) * size, cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        return;
    }
    if (size > res_size_) {
        stored_ = 0;
        res_size_ = size;
        res_count_ = 0;
        truncated_ = false;
    }
    if (size > best_) best_ = size;
    const int64_t stored = stored_;
    // stored list capacity: max_cliques, and never more rows than a quarter of the budget holds
    const int64_t store_cap = o_.max_cliques > 0 ? std::min<int64_t>(o_.max_cliques, stage_max_rows_) : stage_max_rows_;
    const int64_t want = std::min<int64_t>(cnt, std::max<int64_t>(store_cap - stored, 0));
    int64_t &cap = kind ? a.clq_cap : a.leaf_cap;
    if (want > cap) {  // staging too small: grow and replay the count pass (idempotent)
        (kind ? cstage_rows_ : stage_rows_) = want;
        stage.ensure((size_t)want * std::max<int32_t>(g_->max_out + 2, 2));
        (kind ? a.clq_rows : a.leaf_rows) = stage.get();
        cap = want;
        reset_leaf_counters();
        launch_expand(a, false, s_);
        ++kernels_;
        if (kind == 1) materialize_pairs(a);
        stream_sync(s_);
    }
    const int64_t take = std::min<int64_t>(want, cap);
    if (take > 0) {  // append to the device store (grown with copy; read out once at the end)
        const size_t need = (size_t)(stored + take) * size;
        if (g_->store.n < need) {
            DevBuf<int32_t> bigger(std::max(need, g_->store.n * 2));
            if (stored)
                MCE_CUDA(cudaMemcpyAsync(bigger.get(), g_->store.get(), sizeof(int32_t) * stored * size,
                                         cudaMemcpyDeviceToDevice, s_));
            stream_sync(s_);  // the old block goes back to the cache only when unused
            g_->store = std::move(bigger);
        }
        MCE_CUDA(cudaMemcpyAsync(g_->store.get() + (size_t)stored * size, stage.get(),
                                 sizeof(int32_t) * take * size, cudaMemcpyDeviceToDevice, s_));
        stored_ += take;
    }
    if (take < cnt) truncated_ = true;
    res_count_ += cnt;
}

// Small-frontier fused levels (expand_small): consecutive tiny levels in one
// launch; the host then continues with whatever the kernel hands back.
bool Engine::run_small(int32_t k, const Level &L) {
    const Arena::Mark mark = arena_.mark();
    const int64_t scratch_bytes = std::min<int64_t>((int64_t)(arena_.avail() / 2), 256ll << 20);
    if (scratch_bytes < (16ll << 20)) return false;
    uint8_t *scratch = arena_.alloc<uint8_t>(scratch_bytes);
    SmallOut *dout = arena_.alloc<SmallOut>(1);
    ExpandArgs a{};
    a.P = L.P;
    a.slot = L.slot;
    a.parent = L.parent;
    a.vloc = L.vloc;
    a.begin = 0;
    a.end = L.count;
    a.k = k;
    a.need = need();
    a.bound = o_.bound;
    a.Wp = L.W;
    a.Ps = L.Ps > 0 ? L.Ps : L.W;
    a.Wa = W_;
    a.Wc = L.W;
    a.roots = roots_;
    a.adj = adj_;
    a.ocol = vtab_;
    a.order = g_->vid.get();
    a.prefix = prefix_;
    a.k0 = k0_;
    a.maxbit = maxbit_;
    leaf_args(a);
    a.chain = chain_dev_;
    reset_leaf_counters();
    const int t = clock_.start(1);
    launch_expand_small(a, scratch, scratch_bytes, dout, chain_dev_, s_);
    clock_.stop(t);
    ++kernels_;
    SmallOut *h = g_->host.get<SmallOut>(1);
    MCE_CUDA(cudaMemcpyAsync(h, dout, sizeof(SmallOut), cudaMemcpyDeviceToHost, s_));
    stream_sync(s_);
    if (h->levels == 0) {
        arena_.reset(mark);
        return false;
    }
    const SmallOut o = *h;  // the pinned staging is reused by the calls below
    if ((int64_t)level_entries_.size() < k + o.levels) level_entries_.resize(k + o.levels, 0);
    for (int64_t i = 0; i < o.levels; ++i) level_entries_[k + i] += o.level_n[i];
    if (o_.verbose > 0)
        fprintf(stderr, "[mce] fused levels k=%d..%lld entries=%lld -> children=%lld leaves=%lld status=%lld\n", k,
                (long long)(k + o.levels - 1), (long long)L.count, (long long)o.children, (long long)o.leaves,
                (long long)o.status);
    if (o_.verbose > 1)
        fprintf(stderr, "[mce]   cycles: setup %lld staging %lld entry0 %lld (colouring %lld completions %lld branching %lld, %lld vertices) wait %lld tail %lld\n",
                o.prof[0], o.prof[1], o.prof[2], o.prof[6], o.prof[7], o.prof[8], o.prof[9], o.prof[3], o.prof[4]);
    if (o.leaves > 0 || o.cliques > 0) {  // leaves of size k_next / completions of size need, last level
        ExpandArgs la = a;
        la.P = o.inP;
        la.slot = o.inslot;
        la.parent = o.inparent;
        la.vloc = o.invloc;
        la.end = o.inN;
        la.k = (int32_t)o.k_next - 1;
        la.Wp = la.Wc = (int32_t)o.inW;
        la.Ps = (int32_t)o.inPs;
        la.counts = arena_.alloc<int32_t>(o.inN);  // for a count-pass replay if the staging must grow
        handle_leaves((int32_t)o.k_next, o.leaves, la, 0);
        if (o.cliques > 0 && (o.leaves == 0 || (!find_one_ && la.need == (int32_t)o.k_next)))
            handle_leaves(la.need, o.cliques, la, 1);
    }
    sync_bound(true);
    if (o.status == 1 && o.children > 0) {
        Level C;
        C.count = o.children;
        C.W = (int32_t)o.Wc;
        C.Ps = (int32_t)o.Ps;
        C.P = o.P;
        C.slot = o.slot;
        C.parent = o.parent;
        C.vloc = o.vloc;
        process((int32_t)o.k_next, C);
    }
    arena_.reset(mark);
    return true;
}

// Re-rooting (expand.cuh launch_reroot_build): the candidates of a wide level
// (W >= reroot_min_w_ words, e.g. R-MAT scale 26's 2048-4096-vertex roots)
// whose sets hold at most 1024 vertices become roots of their own over P,
// grouped by the width of |P|; each group is processed as a window of its own
// (level k, the same candidates) at that width.  Candidates with larger sets
// stay in the old space.  Returns false (nothing done) when the derived arrays
// would not fit half of the free budget.
bool Engine::reroot(int32_t k, const Level &L) {
    const int64_t N = L.count;
    if (N <= 0) return false;
    const Arena::Mark mark = arena_.mark();
    const int32_t Ps = L.Ps > 0 ? L.Ps : L.W;
    int32_t *Lp = arena_.alloc<int32_t>(N);
    int32_t *cls = arena_.alloc<int32_t>(N);
    int64_t *hist = arena_.alloc<int64_t>(kMaxClass + 1);
    MCE_CUDA(cudaMemsetAsync(hist, 0, sizeof(int64_t) * (kMaxClass + 1), s_));
    launch_reroot_sizes(L.P, Ps, L.W, N, Lp, cls, hist, s_);
    int64_t *hh = g_->host.get<int64_t>(kMaxClass + 1);
    MCE_CUDA(cudaMemcpyAsync(hh, hist, sizeof(int64_t) * (kMaxClass + 1), cudaMemcpyDeviceToHost, s_));
    stream_sync(s_);
    kernels_ += 1;
    std::vector<int64_t> counts(hh, hh + kMaxClass + 1);
    // derived bytes: per re-rooted candidate L' (4 + 8 Wn) + 8 Wn + ~64; bound it by the sizes' upper end
    int64_t need_bytes = 0, moved = 0;
    for (int c = 0; c <= 4 && c <= kMaxClass; ++c) {
        const int64_t Wn = 1ll << c;
        need_bytes += counts[c] * (64 * Wn * (4 + 8 * Wn) + 8 * Wn + 64 + 4 * k);
        moved += counts[c];
    }
    if (moved == 0 || need_bytes > (int64_t)(arena_.avail() / 4)) {  // (the subtrees below need the rest)
        arena_.reset(mark);
        return false;
    }
    if ((int64_t)level_entries_.size() <= k) level_entries_.resize(k + 1, 0);
    // the saved window state (the caller's siblings continue in the old space)
    const RootInfo *sroots = roots_;
    const uint64_t *sadj = adj_;
    const int32_t *svtab = vtab_, *sprefix = prefix_;
    const int32_t sk0 = k0_, sW = W_;
    const int64_t snroots = nroots_;
    int32_t *flag = arena_.alloc<int32_t>(N);
    int64_t *pos = arena_.alloc<int64_t>(N + 1);
    int64_t *tmp = arena_.alloc<int64_t>(scan_tmp_items(N));
    ExpandArgs ra{};
    ra.P = L.P;
    ra.slot = L.slot;
    ra.Wp = L.W;
    ra.Ps = Ps;
    ra.Wa = W_;
    ra.k = k;
    ra.roots = roots_;
    ra.adj = adj_;
    ra.ocol = vtab_;
    ra.order = g_->vid.get();
    ra.chain = chain_dev_;
    ra.prefix = prefix_;
    ra.k0 = k0_;
    if (k + 2 > chain_cap_) fail(MCE_ERR_INVALID, "clique depth above the supported maximum");
    const LevelLink link{L.parent, L.vloc};  // the candidates' own level (read-out of their prefixes)
    for (int c = 0; c <= kMaxClass; ++c) {
        if (counts[c] == 0) continue;
        const Arena::Mark cmark = arena_.mark();
        const int64_t cnt = counts[c];
        int32_t *list = arena_.alloc<int32_t>(cnt);
        launch_flag_eq(N, cls, c, flag, s_);
        exclusive_scan_i32(flag, pos, N, tmp, s_);
        launch_compact(N, flag, pos, list, s_);
        kernels_ += 5;
        if (c > 4) {  // sets above 1024 vertices: the old space, at the old width
            Level O;
            O.count = cnt;
            O.W = L.W;
            O.P = arena_.alloc<uint64_t>(cnt * L.W);
            O.slot = arena_.alloc<int32_t>(cnt);
            O.parent = arena_.alloc<int32_t>(cnt);
            O.vloc = arena_.alloc<int32_t>(cnt);
            launch_gather_level(N, flag, pos, L.W, Ps, L.P, L.slot, L.parent, L.vloc, O.P, O.slot, O.parent, O.vloc, s_);
            kernels_ += 1;
            const int32_t saved = no_reroot_level_;
            no_reroot_level_ = k;  // (no second attempt on these)
            level_entries_[k] -= cnt;  // (counted again by process)
            process(k, O);
            no_reroot_level_ = saved;
            arena_.reset(cmark);
            continue;
        }
        const int Wn = 1 << c;
        int32_t *lens = arena_.alloc<int32_t>(cnt);
        int64_t *voff = arena_.alloc<int64_t>(cnt + 1);
        int64_t *tmp2 = arena_.alloc<int64_t>(scan_tmp_items(cnt));
        launch_gather_i32(Lp, list, cnt, lens, s_);
        exclusive_scan_i32(lens, voff, cnt, tmp2, s_);
        int64_t *hv = g_->host.get<int64_t>(1);
        MCE_CUDA(cudaMemcpyAsync(hv, voff + cnt, sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        const int64_t total = hv[0];
        int32_t *nV = arena_.alloc<int32_t>(total);
        uint64_t *nA = arena_.alloc<uint64_t>(total * Wn);
        RootInfo *nroots = arena_.alloc<RootInfo>(cnt);
        int32_t *nprefix = arena_.alloc<int32_t>(cnt * k);
        Level D;
        D.count = cnt;
        D.W = Wn;
        D.P = arena_.alloc<uint64_t>(cnt * Wn);
        D.slot = arena_.alloc<int32_t>(cnt);
        D.parent = arena_.alloc<int32_t>(cnt);
        D.vloc = arena_.alloc<int32_t>(cnt);
        // (a previous group's process(k, ...) replaced chain[k]: the prefixes read the candidates' own links)
        MCE_CUDA(cudaMemcpyAsync(chain_dev_ + k, &link, sizeof(link), cudaMemcpyHostToDevice, s_));
        const int tcl = clock_.start(3);
        const double bms = timed_step(s_, o_.verbose > 1, [&] {
            launch_reroot_build(ra, list, cnt, voff, Wn, nV, nA, nroots, D.P, D.slot, D.parent, D.vloc, nprefix, s_);
        });
        clock_.stop(tcl);
        if (o_.verbose > 1)
            fprintf(stderr, "[mce] re-root build k=%d Wn=%d candidates=%lld: %.3f ms\n", k, (int)Wn, (long long)cnt, bms);
        kernels_ += 4;
        roots_ = nroots;
        adj_ = nA;
        vtab_ = nV;
        prefix_ = nprefix;
        k0_ = k;
        W_ = Wn;
        nroots_ = cnt;
        level_entries_[k] -= cnt;  // (counted again by process)
        const int32_t saved = no_reroot_level_;
        no_reroot_level_ = k;  // the derived level itself is not re-rooted again (deeper levels may be)
        process(k, D);
        no_reroot_level_ = saved;
        roots_ = sroots;
        adj_ = sadj;
        vtab_ = svtab;
        prefix_ = sprefix;
        k0_ = sk0;
        W_ = sW;
        nroots_ = snroots;
        arena_.reset(cmark);
    }
    level_entries_[k] += N;
    arena_.reset(mark);
    return true;
}

void Engine::process(int32_t k, const Level &L) {
    if (entry_shard_ && !split_ && k >= o_.shard_depth) {  // deal this level's entries by path hash
        if (k + 2 > chain_cap_) fail(MCE_ERR_INVALID, "clique depth above the supported maximum");
        LevelLink link{L.parent, L.vloc};
        MCE_CUDA(cudaMemcpyAsync(chain_dev_ + k, &link, sizeof(link), cudaMemcpyHostToDevice, s_));
        const Arena::Mark mark = arena_.mark();
        const int64_t N = L.count;
        const int32_t Ps = L.Ps > 0 ? L.Ps : L.W;
        int32_t *flag = arena_.alloc<int32_t>(N);
        int64_t *pos = arena_.alloc<int64_t>(N + 1);
        int64_t *tmp = arena_.alloc<int64_t>(scan_tmp_items(N));
        ExpandArgs sa{};
        sa.roots = roots_;
        sa.slot = L.slot;
        sa.chain = chain_dev_;
        sa.ocol = vtab_;
        sa.order = g_->vid.get();
        sa.prefix = prefix_;
        sa.k0 = k0_;
        launch_shard_flags(sa, N, k, (int32_t)offset_, (int32_t)stride_, flag, s_);
        exclusive_scan_i32(flag, pos, N, tmp, s_);
        int64_t *h = g_->host.get<int64_t>(1);
        MCE_CUDA(cudaMemcpyAsync(h, pos + N, sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        kernels_ += 4;
        const int64_t mine = h[0];
        Level F;
        F.count = mine;
        F.W = L.W;
        F.P = arena_.alloc<uint64_t>(mine * L.W);
        F.slot = arena_.alloc<int32_t>(mine);
        F.parent = arena_.alloc<int32_t>(mine);
        F.vloc = arena_.alloc<int32_t>(mine);
        launch_gather_level(N, flag, pos, L.W, Ps, L.P, L.slot, L.parent, L.vloc, F.P, F.slot, F.parent, F.vloc,
                            s_);
        ++kernels_;
        split_ = true;
        if (mine > 0) process(k, F);
        split_ = false;
        arena_.reset(mark);
        return;
    }
    if (k >= 2 && k != no_reroot_level_ && reroot_min_w_ > 0 && L.W >= reroot_min_w_ && !o_.no_reroot &&
        reroot(k, L))
        return;
    const bool pre_split = entry_shard_ && !split_;  // fused tiny levels would run past the split depth
    if (!pre_split && !o_.no_fused_levels && L.count <= kSmallMax && L.W <= 4 && run_small(k, L)) return;
    if ((int64_t)level_entries_.size() <= k) level_entries_.resize(k + 1, 0);
    level_entries_[k] += L.count;
    if (k + 2 > chain_cap_) fail(MCE_ERR_INVALID, "clique depth above the supported maximum");
    LevelLink link{L.parent, L.vloc};
    MCE_CUDA(cudaMemcpyAsync(chain_dev_ + k, &link, sizeof(link), cudaMemcpyHostToDevice, s_));

    const Arena::Mark mark = arena_.mark();
    const int64_t N = L.count;
    int32_t *counts = arena_.alloc<int32_t>(N);
    int64_t *offs = arena_.alloc<int64_t>(N + 1);
    int64_t *tmp = arena_.alloc<int64_t>(scan_tmp_items(N));
    int64_t *chunk = arena_.alloc<int64_t>(4);

    ExpandArgs a{};
    a.P = L.P;
    a.slot = L.slot;
    a.parent = L.parent;
    a.vloc = L.vloc;
    a.begin = 0;
    a.end = N;
    a.k = k;
    a.need = need();
    a.bound = o_.bound;
    a.Wp = L.W;
    a.Ps = L.Ps > 0 ? L.Ps : L.W;
    a.Wa = W_;
    a.Wc = L.W;
    a.roots = roots_;
    a.adj = adj_;
    a.ocol = vtab_;
    a.order = g_->vid.get();
    a.prefix = prefix_;
    a.k0 = k0_;
    a.counts = counts;
    a.maxbit = maxbit_;
    leaf_args(a);
    a.chain = chain_dev_;
    // shared-memory count pass (expand_smem): the level's entries grouped by
    // root slot so a block stages one root's matrix per run of its candidates
    // (only when a root has many candidates on average: one entry per root, as at
    // level 1, gains nothing from staging 64 W rows and loses the L2's parallelism)
    // A level of at most one entry per SM is the other case: every candidate is a
    // long serial colouring chain with nothing to overlap it, and a block of its
    // own turns the chain's row reads from L2 into shared-memory hits.
    const bool many_per_root = N >= smem_min_n_ && N >= smem_per_root_ * nroots_;
    const bool few_chains = N <= num_sms();
    if (!o_.no_smem_expand && smem_width(L.W) && L.W >= smem_min_w_ && nroots_ > 0 && (many_per_root || few_chains)) {
        int32_t *hist = arena_.alloc<int32_t>(nroots_);
        int64_t *hoffs = arena_.alloc<int64_t>(nroots_ + 1);
        int64_t *htmp = arena_.alloc<int64_t>(scan_tmp_items(nroots_));
        int32_t *perm = arena_.alloc<int32_t>(N);
        launch_group_by_slot(L.slot, N, (int32_t)nroots_, hist, hoffs, htmp, perm, s_);
        kernels_ += 5;
        a.perm = perm;
        a.chunk_ctr = chunk_ctr_;
        a.universal = 0;  // (the lockstep count pass colours every candidate: the write pass must too)
    }

    a.chunk_ctr = chunk_ctr_;  // (dynamic work counter of the shared-memory and wide count passes)
    if (!a.perm && L.W >= wide_min_w() && L.W <= 64) {
        // expand_wide's colouring orders (64 W u16 per tile): a workspace kept on the graph
        // (like the leaf staging, outside the frontier budget); the launch takes as many
        // blocks as it holds, at most 64 MB
        const int64_t want = std::min<int64_t>((int64_t)num_sms() * 8 * 32 * 64 * L.W, 32ll << 20);
        g_->wide.ensure((size_t)want);
        a.wscratch = g_->wide.get();
        a.wscratch_n = (int64_t)g_->wide.n;
    }

    // Fused count + write: the children are written by the count pass into
    // arrays sized for half of the free budget; if they fit they are compacted
    // and the next level starts without a scan or a write pass.
    const int64_t per_child = 8 * L.W + 12;
    Arena::Mark fmark = arena_.mark();
    bool fused = false;
    int64_t fcap = 0;
    uint64_t *fP = nullptr;
    int32_t *fslot = nullptr, *fparent = nullptr, *fvloc = nullptr;
    if (!o_.no_fused_expand) {
        // capacity: half of the free budget, at most 16 children per entry (+1M);
        // a level that branches wider overflows into scan + chunked writes
        fcap = std::min<int64_t>((int64_t)(arena_.avail() / 2) / (per_child + 64), 16 * N + (1 << 20));
        // a power of two: budget jitter between calls then asks for the same
        // sizes, so the arena's kept segments are reused (no re-allocation)
        int64_t p2 = 1;
        while (p2 * 2 <= fcap) p2 <<= 1;
        fcap = p2;
        if (fcap >= 1024) {
            fP = arena_.alloc<uint64_t>(fcap * L.W, &fmark);
            fslot = arena_.alloc<int32_t>(fcap);
            fparent = arena_.alloc<int32_t>(fcap);
            fvloc = arena_.alloc<int32_t>(fcap);
            fused = true;
            a.fused = 1;
            a.out_count = out_count_;
            a.out_cap = fcap;
            a.cP = fP;
            a.cslot = fslot;
            a.cparent = fparent;
            a.cvloc = fvloc;
        }
    }

    // misc[0..4] = leaf total, leaf slot, completion total, completion slot, maxbit (-1); misc[5] = fused children
    reset_leaf_counters();
    MCE_CUDA(cudaMemsetAsync(maxbit_, 0xff, 2 * sizeof(int32_t), s_));
    if (fused) MCE_CUDA(cudaMemsetAsync(out_count_, 0, sizeof(unsigned long long), s_));
    launch_timed(a, false);
    kernels_ += 1;
    if (!fused) {
        exclusive_scan_i32(counts, offs, N, tmp, s_);
        kernels_ += 2;
    }
    int64_t *h = g_->host.get<int64_t>(8);
    if (!fused) MCE_CUDA(cudaMemcpyAsync(h, offs + N, sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
    MCE_CUDA(cudaMemcpyAsync(h + 1, leaf_total_, 6 * sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
    stream_sync(s_);
    const int64_t total = fused ? h[6] : h[0];
    const unsigned long long leaves = (unsigned long long)h[1];
    const int64_t completions = h[3];
    const int32_t maxbit = (int32_t)(uint32_t)(uint64_t)h[5];
    const int32_t maxub = (int32_t)(uint32_t)((uint64_t)h[5] >> 32);  // deepest reachable level
    // children's candidate sets only use bits <= maxbit: shrink their stride
    // (power of two, so the kernels stay specialised)
    int32_t Wc = 1;
    while (Wc * 64 <= maxbit && Wc < L.W) Wc <<= 1;
    a.Wc = Wc;
    if (o_.verbose > 0)
        fprintf(stderr, "[mce] level k=%d entries=%lld W=%d children=%lld leaves=%llu completions=%lld need=%d%s%s\n",
                k, (long long)N, L.W, (long long)total, leaves, (long long)completions, a.need,
                fused ? (total <= fcap ? " fused" : " fused-overflow") : "", a.perm ? " smem" : "");
    const int32_t need_counted = a.need;
    a.fused = 0;  // a count-pass replay (staging growth) must not write children again
    if (leaves) handle_leaves(k + 1, (int64_t)leaves, a, 0);
    if (completions > 0 && (leaves == 0 || (!find_one_ && need_counted == k + 1)))
        handle_leaves(need_counted, completions, a, 1);

    if (fused && total <= fcap) {
        count_bytes_ += (double)total * (8.0 * L.W + 12.0);  // the children the fused pass wrote
        Level C;
        C.count = total;
        C.W = Wc;
        C.Ps = L.W;
        if (total > 0) {
            // compact: slot/parent/vloc go to a temporary behind the fcap-sized
            // arrays, then to tight arrays right behind P (P stays in place);
            // the tight arrays end before the temporary starts (total <= fcap)
            int32_t *tmp3 = arena_.alloc<int32_t>(3 * total);
            MCE_CUDA(cudaMemcpyAsync(tmp3, fslot, sizeof(int32_t) * total, cudaMemcpyDeviceToDevice, s_));
            MCE_CUDA(cudaMemcpyAsync(tmp3 + total, fparent, sizeof(int32_t) * total, cudaMemcpyDeviceToDevice, s_));
            MCE_CUDA(cudaMemcpyAsync(tmp3 + 2 * total, fvloc, sizeof(int32_t) * total, cudaMemcpyDeviceToDevice,
                                     s_));
            arena_.reset(fmark);
            C.P = arena_.alloc<uint64_t>(total * L.W);  // == fP
            C.slot = arena_.alloc<int32_t>(total);
            C.parent = arena_.alloc<int32_t>(total);
            C.vloc = arena_.alloc<int32_t>(total);
            MCE_CUDA(cudaMemcpyAsync(C.slot, tmp3, sizeof(int32_t) * total, cudaMemcpyDeviceToDevice, s_));
            MCE_CUDA(cudaMemcpyAsync(C.parent, tmp3 + total, sizeof(int32_t) * total, cudaMemcpyDeviceToDevice, s_));
            MCE_CUDA(cudaMemcpyAsync(C.vloc, tmp3 + 2 * total, sizeof(int32_t) * total, cudaMemcpyDeviceToDevice,
                                     s_));
            if (C.P != fP) fail(MCE_ERR_INVALID, "internal: fused level moved");
        }
        sync_bound(true);
        if (total > 0) process(k + 1, C);
        arena_.reset(mark);
        return;
    }
    if (fused) {  // overflow: the children did not fit; scan the counts and write in chunks
        arena_.reset(fmark);
        exclusive_scan_i32(counts, offs, N, tmp, s_);
        kernels_ += 2;
    }

    const int64_t per_child2 = 8 * Wc + 12 + 12 + 16;
    // When the children do not fit they are produced in chunks.  Each chunk may
    // take 1/(levels still reachable below it + 1) of the free arena, so a
    // frontier that keeps growing for many levels (R-MAT: 2x per level over the
    // last ~30 levels) is chunked evenly instead of halving the budget per level.
    const int64_t depth_left = std::max<int64_t>(1, (int64_t)maxub - (k + 1));
    int64_t a0 = 0;
    while (total > 0 && a0 < N) {
        // kLevelReserve stays free for the fixed small allocations of the levels
        // below (every arena allocation is rounded to kAlign bytes, which the
        // per-child share does not cover: under a few-MB budget a deep chain of
        // chunked levels otherwise ends on a 256-byte allocation with nothing left)
        const int64_t usable = std::max<int64_t>(0, (int64_t)arena_.avail() - kLevelReserve);
        const int64_t share = total * per_child2 <= usable / 2 ? 2 : depth_left + 1;
        const int64_t cap = (usable / share) / per_child2;
        int64_t b, cnt, base;
        if (a0 == 0 && total <= cap) {
            b = N;
            cnt = total;
            base = 0;
        } else {
            launch_find_chunk_end(offs, a0, N, cap, chunk, s_);
            ++kernels_;
            int64_t *hc = g_->host.get<int64_t>(3);
            MCE_CUDA(cudaMemcpyAsync(hc, chunk, 3 * sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
            stream_sync(s_);
            b = hc[0];
            cnt = hc[1];
            base = hc[2];
            if (b == a0 && share > 2) {
                // one candidate's children exceed this level's share: let that chunk
                // take half of what is left (the levels below it still get the rest)
                launch_find_chunk_end(offs, a0, N, (usable / 2) / per_child2, chunk, s_);
                ++kernels_;
                MCE_CUDA(cudaMemcpyAsync(hc, chunk, 3 * sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
                stream_sync(s_);
                b = hc[0];
                cnt = hc[1];
                base = hc[2];
            }
            if (b == a0)
                fail(MCE_ERR_BUDGET, "the children of one candidate at level " + std::to_string(k) +
                                         " exceed the frontier budget");
        }
        const Arena::Mark cmark = arena_.mark();
        Level C;
        C.count = cnt;
        C.W = Wc;
        C.P = arena_.alloc<uint64_t>(cnt * Wc);
        C.slot = arena_.alloc<int32_t>(cnt);
        C.parent = arena_.alloc<int32_t>(cnt);
        C.vloc = arena_.alloc<int32_t>(cnt);
        ExpandArgs w = a;
        w.perm = nullptr;
        w.begin = a0;
        w.end = b;
        w.offsets = offs;
        w.out_base = base;
        w.cP = C.P;
        w.cslot = C.slot;
        w.cparent = C.parent;
        w.cvloc = C.vloc;
        launch_timed(w, true);
        sync_bound(true);
        if (cnt > 0) process(k + 1, C);
        arena_.reset(cmark);
        a0 = b;
    }
    arena_.reset(mark);
}

// W == 1 roots: the fused root level (roots.cu), then levels >= 2 as usual
void Engine::do_class_w1(const int32_t *list, int64_t count) {
    // the class list holds this shard's roots only (classify_roots deals them)
    const int64_t mine = count;
    if (mine <= 0) return;
    W_ = 1;
    const int32_t *base = list;
    unsigned long long *ctr = arena_.alloc<unsigned long long>(8);
    // per candidate row: adjacency word + one level-2 entry (P, slot, parent, vloc)
    const int64_t row_bytes = 8 + 8 + 12;
    const int64_t per_root = sizeof(RootInfo) + 64;
    // Sparse orientation (every |N+(r)| <= 4, no window requested): when
    // max_out rows per root fit, the whole class is one window sized by that
    // bound, with no row-count pass, scan or read-back
    const bool one_window = o_.window <= 0 && g_->max_out <= 4 &&
                            (int64_t)(arena_.avail() / 3) >= mine * (per_root + row_bytes * std::max(g_->max_out, 1));
    int64_t *prefix = nullptr, *win = nullptr;
    if (!one_window) {
        int32_t *len = arena_.alloc<int32_t>(mine);
        prefix = arena_.alloc<int64_t>(mine + 1);
        int64_t *tmp = arena_.alloc<int64_t>(scan_tmp_items(mine));
        win = arena_.alloc<int64_t>(2);
        launch_root_lengths(base, mine, 1, g_->orp.get(), len, s_);
        exclusive_scan_i32(len, prefix, mine, tmp, s_);
        kernels_ += 4;
    }
    int64_t hi = mine;
    while (hi > 0) {
        const Arena::Mark mark = arena_.mark();
        int64_t lo = 0, rows = 0;
        if (one_window) {
            rows = mine * std::max(g_->max_out, 1);
        } else {
            const int64_t room = (int64_t)(arena_.avail() / 3);
            const int64_t maxw = o_.window > 0 ? o_.window : hi;
            launch_find_window(prefix, hi, std::max<int64_t>(0, hi - maxw), room, row_bytes, per_root, win, s_);
            ++kernels_;
            int64_t *hw = g_->host.get<int64_t>(2);
            MCE_CUDA(cudaMemcpyAsync(hw, win, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
            stream_sync(s_);
            lo = hw[0];
            rows = hw[1];
        }
        const int64_t nw = hi - lo;
        RootArgs ra{};
        ra.list = base + lo;
        ra.count = nw;
        ra.stride = 1;
        ra.orp = g_->orp.get();
        ra.ocol = g_->ocol.get();
        ra.ocol4 = g_->have_ocol4 ? g_->ocol4.get() : nullptr;
        ra.order = g_->vid.get();
        ra.need = need();
        ra.bound = o_.bound;
        ra.roots = arena_.alloc<RootInfo>(nw);
        ra.adj = arena_.alloc<uint64_t>(rows);
        ra.cP = arena_.alloc<uint64_t>(rows);
        ra.cslot = arena_.alloc<int32_t>(rows);
        ra.cparent = arena_.alloc<int32_t>(rows);
        ra.cvloc = arena_.alloc<int32_t>(rows);
        ra.ctr = ctr;
        ra.leaf_rows = g_->stage.get();
        ra.leaf_cap = stage_rows_;
        unsigned long long *hc = nullptr;
        for (int attempt = 0; attempt < 2; ++attempt) {
            MCE_CUDA(cudaMemsetAsync(ctr, 0, 8 * sizeof(unsigned long long), s_));
            const int t = clock_.start(2);
            // the sparse kernel takes 32-bit offsets into the oriented CSR
            launch_root_expand_w1(ra, g_->nnz / 2 < INT32_MAX ? g_->max_out : 64, s_);
            clock_.stop(t);
            ++kernels_;
            ++root_launches_;
            hc = g_->host.get<unsigned long long>(8);
            MCE_CUDA(cudaMemcpyAsync(hc, ctr, 8 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s_));
            stream_sync(s_);
            const int64_t leaves = (int64_t)hc[3];
            if (attempt == 0 && leaves > ra.leaf_cap && !find_one_) {
                // staging too small for the size-2 leaves: grow and replay (counters reset)
                int64_t want = std::min<int64_t>(leaves, stage_max_rows_);
                if (o_.max_cliques > 0) want = std::min<int64_t>(want, o_.max_cliques);
                if (want > ra.leaf_cap) {
                    stage_rows_ = want;
                    g_->stage.ensure((size_t)want * std::max<int32_t>(g_->max_out + 2, 2));
                    ra.leaf_rows = g_->stage.get();
                    ra.leaf_cap = want;
                    continue;
                }
            }
            break;
        }
        root_bytes_ += (double)hc[4];
        if ((int64_t)level_entries_.size() <= 1) level_entries_.resize(2, 0);
        level_entries_[1] += nw;
        const int64_t leaves = (int64_t)hc[3];
        if (leaves > 0) {
            ExpandArgs la{};
            la.k = 1;
            la.ocol = g_->ocol.get();
            la.order = g_->vid.get();
            leaf_args(la);
            la.leaf_rows = ra.leaf_rows;
            la.leaf_cap = ra.leaf_cap;
            handle_leaves(2, leaves, la, 0);
        }
        const int64_t entries = (int64_t)hc[2];
        if (o_.verbose > 0)
            fprintf(stderr, "[mce] roots=%lld survivors=%llu level2=%lld leaves=%lld need=%d\n", (long long)nw,
                    hc[0], (long long)entries, (long long)leaves, need());
        if (entries > 0) {
            roots_ = ra.roots;
            adj_ = ra.adj;
            nroots_ = nw;
            vtab_ = g_->ocol.get();
            prefix_ = nullptr;
            k0_ = 0;
            Level L2;
            L2.count = entries;
            L2.W = 1;
            L2.P = ra.cP;
            L2.slot = ra.cslot;
            L2.parent = ra.cparent;
            L2.vloc = ra.cvloc;
            process(2, L2);
        }
        sync_bound(true);
        arena_.reset(mark);
        hi = lo;
    }
}

void Engine::do_class(int32_t cls, const int32_t *list, int64_t count) {
    if (cls == 0 && !o_.legacy_roots) {
        do_class_w1(list, count);
        return;
    }
    // the class list holds this shard's roots only (classify_roots deals them)
    const int64_t mine = count;
    if (mine <= 0) return;
    W_ = 1 << cls;
    const int32_t *base = list;
    // adjacency rows per root -> prefix; it stays on the device and windows
    // are cut there (one scalar read-back per window)
    int32_t *len = arena_.alloc<int32_t>(mine);
    int64_t *prefix = arena_.alloc<int64_t>(mine + 1);
    int64_t *tmp = arena_.alloc<int64_t>(scan_tmp_items(mine));
    int64_t *win = arena_.alloc<int64_t>(2);
    launch_root_lengths(base, mine, 1, g_->orp.get(), len, s_);
    exclusive_scan_i32(len, prefix, mine, tmp, s_);
    kernels_ += 4;
    const int64_t per_root = sizeof(RootInfo) + 8 * W_ + 12 + 64;
    // windows from the highest ranks down (densest cores first)
    int64_t hi = mine;
    while (hi > 0) {
        const Arena::Mark mark = arena_.mark();
        const int64_t room = (int64_t)(arena_.avail() / 4);
        const int64_t maxw = o_.window > 0 ? o_.window : hi;
        // smallest lo >= hi - maxw whose rows fit a quarter of the free budget (at least one root)
        launch_find_window(prefix, hi, std::max<int64_t>(0, hi - maxw), room, 8 * W_, per_root, win, s_);
        ++kernels_;
        int64_t *hw = g_->host.get<int64_t>(2);
        MCE_CUDA(cudaMemcpyAsync(hw, win, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        const int64_t lo = hw[0], rows = hw[1];
        const int64_t nw = hi - lo;
        RootInfo *roots = arena_.alloc<RootInfo>(nw);
        uint64_t *adj = arena_.alloc<uint64_t>(rows * W_);
        launch_make_roots(base + lo, nw, 1, W_, g_->orp.get(), prefix + lo, roots, s_);
        const int tcl = clock_.start(4);
        const double bms = timed_step(s_, o_.verbose > 1, [&] {
            launch_build_adj(roots, nw, W_, g_->orp.get(), g_->ocol.get(), adj, rows * W_, s_, build_bytes_);
        });
        ++build_launches_;
        clock_.stop(tcl);
        if (o_.verbose > 1)
            fprintf(stderr, "[mce] root build W=%d roots=%lld rows=%lld: %.3f ms\n", W_, (long long)nw, (long long)rows,
                    bms);
        kernels_ += 2;
        roots_ = roots;
        adj_ = adj;
        nroots_ = nw;
        vtab_ = g_->ocol.get();
        prefix_ = nullptr;
        k0_ = 0;
        Level L1;
        L1.count = nw;
        L1.W = W_;
        L1.P = arena_.alloc<uint64_t>(nw * W_);
        L1.slot = arena_.alloc<int32_t>(nw);
        L1.parent = arena_.alloc<int32_t>(nw);
        L1.vloc = arena_.alloc<int32_t>(nw);
        launch_init_level1(roots, nw, W_, L1.P, L1.slot, L1.parent, L1.vloc, s_);
        ++kernels_;
        process(1, L1);
        sync_bound(true);
        arena_.reset(mark);
        hi = lo;
    }
}

mce_result *Engine::run() {
    auto *res = new mce_result();
    using clk = std::chrono::steady_clock;
    const auto h0 = clk::now();
    const int64_t syncs0 = g_syncs;
    auto ms_since = [](clk::time_point t) { return std::chrono::duration<double, std::milli>(clk::now() - t).count(); };
    const int64_t n = g_->n;
    stride_ = o_.shard_count > 1 ? o_.shard_count : 1;
    offset_ = o_.shard_count > 1 ? o_.shard_rank : 0;
    entry_shard_ = stride_ > 1 && o_.shard_depth >= 2;
    if (n == 0) {  // the empty clique is the only clique of the null graph
        res->omega = 0;
        res->count = 1;
        res->stored = 1;
        sync_bound(false);
        return res;
    }
    if (g_->nnz == 0) {  // edgeless: every vertex is a maximum clique
        res->omega = 1;
        for (int64_t v = offset_; v < n; v += stride_) {
            if (find_one_ && !res->rows.empty()) break;
            res->rows.push_back((int32_t)v);
        }
        res->stored = (int64_t)res->rows.size();
        res->count = find_one_ ? 1 : res->stored;
        if (o_.max_cliques > 0 && res->stored > o_.max_cliques) {
            res->rows.resize(o_.max_cliques);
            res->stored = o_.max_cliques;
            res->truncated = 1;
        }
        sync_bound(false);
        return res;
    }
    int heur = o_.heuristic;
    if (find_one_ && heur == 0) heur = 1;  // find-one needs an incumbent clique
    HeuristicResult hr;
    const bool need_pre = !preprocessed(g_, o_.orientation);
    if (!o_.no_overlap && need_pre && (heur == MCE_HEUR_SINGLE_DEGREE || heur == MCE_HEUR_MULTI_DEGREE)) {
        // the degree heuristics read only the CSR: run them on a second stream
        // and host thread while the k-core peel and the orientation run here
        if (!g_->hstream) MCE_CUDA(cudaStreamCreateWithFlags(&g_->hstream, cudaStreamNonBlocking));
        cudaEvent_t ready;
        MCE_CUDA(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
        // KCORE_FIRST (degeneracy orientations): the k-core peel runs alone on the
        // whole GPU first, then the heuristic overlaps only the orientation and
        // uses the core numbers (seeds and candidates of core + 1 < best cannot
        // matter: reading 15); otherwise the heuristic overlaps the peel too
        const bool core_first = KCORE_FIRST && o_.orientation != MCE_ORIENT_DEGREE;
        if (core_first) {
            if (!g_->pre_ev[0]) {
                MCE_CUDA(cudaEventCreate(&g_->pre_ev[0]));
                MCE_CUDA(cudaEventCreate(&g_->pre_ev[1]));
            }
            MCE_CUDA(cudaEventRecord(g_->pre_ev[0], s_));
            g_->pre_started = true;
            kcore(g_);
        }
        MCE_CUDA(cudaEventRecord(ready, s_));  // the CSR (and with core_first the core numbers) is on the device
        std::exception_ptr err;
        double h_heur = 0.0;
        const int dev = g_->device;
        std::thread th([&] {
            try {
                const auto t0 = clk::now();
                MCE_CUDA(cudaSetDevice(dev));
                MCE_CUDA(cudaStreamWaitEvent(g_->hstream, ready, 0));
                hr = run_heuristic(g_, heur, o_.heuristic_runs, (int32_t)offset_, (int32_t)stride_, false, true,
                                   core_first);
                h_heur = ms_since(t0);
            } catch (...) {
                err = std::current_exception();
            }
        });
        // PRE_PRIORITY: the preprocessing runs on a greatest-priority stream, so
        // the orientation's blocks are scheduled ahead of the heuristic's (the
        // heuristic finishes first anyway); events hand the work back to s_
        cudaStream_t user = g_->stream;
        if (PRE_PRIORITY && !g_->pstream) {
            int lo = 0, hi = 0;
            MCE_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
            MCE_CUDA(cudaStreamCreateWithPriority(&g_->pstream, cudaStreamNonBlocking, hi));
        }
        try {
            if (PRE_PRIORITY) {
                MCE_CUDA(cudaStreamWaitEvent(g_->pstream, ready, 0));
                g_->stream = g_->pstream;
            }
            g_->pre_overlapped = !core_first;
            preprocess(g_, o_.orientation);
            g_->pre_overlapped = false;
            if (PRE_PRIORITY) {
                g_->stream = user;
                cudaEvent_t pre_done;
                MCE_CUDA(cudaEventCreateWithFlags(&pre_done, cudaEventDisableTiming));
                MCE_CUDA(cudaEventRecord(pre_done, g_->pstream));
                MCE_CUDA(cudaStreamWaitEvent(user, pre_done, 0));
                cudaEventDestroy(pre_done);  // (released once recorded work completes)
            }
        } catch (...) {
            g_->stream = user;
            g_->pre_overlapped = false;
            th.join();
            cudaEventDestroy(ready);
            throw;
        }
        th.join();
        cudaEventDestroy(ready);
        if (err) std::rethrow_exception(err);
        res->h_pre_ms = ms_since(h0);
        res->t_heur_ms = hr.ms;
        res->h_heur_ms = h_heur;
        res->overlapped = 1;
        kernels_ += g_->kernels;
    } else {
        preprocess(g_, o_.orientation);
        res->h_pre_ms = ms_since(h0);
        const auto h1 = clk::now();
        kernels_ += g_->kernels;
        hr = run_heuristic(g_, heur, o_.heuristic_runs, (int32_t)offset_, (int32_t)stride_, false);
        res->t_heur_ms = hr.ms;
        res->h_heur_ms = ms_since(h1);
    }
    kernels_ += hr.kernels;
    best_ = std::max<int32_t>(hr.omega_bar, 2);
    if (find_one_) {
        res_size_ = hr.omega_bar;
        res_count_ = 1;
        rows_ = hr.clique;
        if (o_.bound_sync) sync_bound(true);
    } else {
        best_ = std::max(best_, o_.lower_bound);
        sync_bound(true);
    }

    // frontier budget: the graph's workspace is reused across calls, so it
    // counts as free memory here
    const auto h2 = clk::now();
    size_t free_b = dev_free_memory();  // (cudaMemGetInfo costs ~1 ms: cached for a second)
    size_t held = dev_cached_bytes();
    for (auto &sg : g_->wsegs) held += sg.n;
    free_b += held;
    // default budget: half of the free device memory; the first segment is
    // sized for a typical run, the rest is only allocated if the frontier needs it
    int64_t budget = o_.budget_bytes > 0 ? o_.budget_bytes : (int64_t)(free_b / 2);
    budget = std::min<int64_t>(budget, (int64_t)(free_b * 0.95));
    const int64_t first = std::min<int64_t>(budget, (int64_t)(1ll << 30) + 48ll * g_->nnz + 64ll * n);
    arena_.init(g_->wsegs, (size_t)budget, (size_t)first);
    // leaf counter + level chain (persistent, g->misc)
    chain_cap_ = 4096;
    g_->misc.ensure(256 + sizeof(LevelLink) * chain_cap_);
    leaf_total_ = reinterpret_cast<unsigned long long *>(g_->misc.get());
    leaf_slot_ = leaf_total_ + 1;
    clq_total_ = leaf_total_ + 2;
    clq_slot_ = leaf_total_ + 3;
    maxbit_ = reinterpret_cast<int32_t *>(leaf_total_ + 4);
    out_count_ = leaf_total_ + 5;
    pair_n_ = leaf_total_ + 6;
    chunk_ctr_ = leaf_total_ + 7;
    build_bytes_ = leaf_total_ + 8;
    MCE_CUDA(cudaMemsetAsync(build_bytes_, 0, sizeof(unsigned long long), s_));
    if (const char *sw = getenv("MCE_SMEM_MIN_W")) smem_min_w_ = atoi(sw);  // tuning hooks (A/B runs)
    if (const char *sn = getenv("MCE_SMEM_MIN_N")) smem_min_n_ = atoll(sn);
    if (const char *sp = getenv("MCE_SMEM_PER_ROOT")) smem_per_root_ = atoll(sp);
    if (const char *rr = getenv("MCE_REROOT_MIN_W")) reroot_min_w_ = atoi(rr);
    pair_cap_ = std::max<int64_t>(4096, (int64_t)g_->pdesc.n / 3);
    g_->pdesc.ensure((size_t)pair_cap_ * 3);
    chain_dev_ = reinterpret_cast<LevelLink *>(g_->misc.get() + 256);
    vtab_ = g_->ocol.get();
    stage_max_rows_ = std::max<int64_t>(1ll << 20, budget / 4 / (4ll * std::max<int32_t>(g_->max_out + 2, 2)));
    // staging rows: whatever the buffers kept from earlier calls hold (a count
    // pass is replayed when the staging is too small, so reuse avoids replays)
    const int64_t row_w = std::max<int32_t>(g_->max_out + 2, 2);
    stage_rows_ = find_one_ ? 1 : std::max<int64_t>(4096, (int64_t)g_->stage.n / row_w);
    g_->stage.ensure((size_t)stage_rows_ * row_w);
    cstage_rows_ = find_one_ ? 1 : std::max<int64_t>(4096, (int64_t)g_->cstage.n / row_w);
    g_->cstage.ensure((size_t)cstage_rows_ * row_w);

    res->h_setup_ms = ms_since(h2);
    const auto h3 = clk::now();
    Timer tt(s_);
    tt.start();
    // roots worth expanding: 1 + |N+(r)| >= need, grouped by candidate-set width class
    {
        const Arena::Mark mark = arena_.mark();
        int32_t *cls = arena_.alloc<int32_t>(n);
        int32_t *flag = arena_.alloc<int32_t>(n);
        int64_t *pos = arena_.alloc<int64_t>(n + 1);
        int64_t *tmp = arena_.alloc<int64_t>(scan_tmp_items(n));
        int64_t *hist = arena_.alloc<int64_t>(kMaxClass + 1);
        MCE_CUDA(cudaMemsetAsync(hist, 0, sizeof(int64_t) * (kMaxClass + 1), s_));
        // root colour filter (colour.cu, reading 14): roots whose
        // out-neighbourhood meets fewer than need - 1 colours of a greedy
        // colouring of the vertices of core >= need - 1 are dropped here
        const uint8_t *rkeep = nullptr;
        int64_t rT = 0;
        if (o_.bound == MCE_BOUND_COLOR && !o_.no_root_colour && g_->max_out >= 64) {
            uint8_t *keepb = arena_.alloc<uint8_t>(n);
            const Arena::Mark cm = arena_.mark();
            int32_t *colr = arena_.alloc<int32_t>(n);
            int64_t *scr = arena_.alloc<int64_t>(4);
            int64_t kept = 0;
            const char *ms = getenv("MCE_ROOT_COLOUR_MIN_S");
            const int tcl = clock_.start(3);
            bool ran = false;
            const double fms = timed_step(s_, o_.verbose > 1, [&] {
                ran = root_colour_filter(g_, need(), ms ? atoll(ms) : kRootColourMinS, keepb, colr, scr, s_, &rT, &kept);
            });
            clock_.stop(tcl);
            if (o_.verbose > 1) fprintf(stderr, "[mce] root colour filter: %.3f ms\n", fms);
            if (ran) {
                rkeep = keepb;
                kernels_ += 4;
                if (o_.verbose > 0)
                    fprintf(stderr, "[mce] root colour filter: %lld vertices of core >= %d, %lld roots kept\n",
                            (long long)(n - rT), need() - 1, (long long)kept);
            }
            arena_.reset(cm);
        }
        // roots are dealt to shards by CSR id (r % shard_count): independent of the
        // lower bound, so ranks whose bounds differ still partition the roots exactly
        launch_classify_roots(n, g_->orp.get(), std::max<int32_t>(need() - 1, 1), entry_shard_ ? 0 : (int32_t)offset_,
                              entry_shard_ ? 1 : (int32_t)stride_, rkeep, rT, cls, hist, s_);
        ++kernels_;
        int64_t *hh = g_->host.get<int64_t>(kMaxClass + 1);
        MCE_CUDA(cudaMemcpyAsync(hh, hist, sizeof(int64_t) * (kMaxClass + 1), cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        if (hh[kMaxClass]) fail(MCE_ERR_INVALID, "out-degree above 16384 after orientation is not supported");
        std::vector<int64_t> counts(hh, hh + kMaxClass);
        std::vector<std::pair<int32_t, int64_t>> classes;
        std::vector<int32_t *> lists;
        for (int32_t c = kMaxClass - 1; c >= 0; --c) {
            if (counts[c] == 0) continue;
            int32_t *list = arena_.alloc<int32_t>(counts[c]);
            launch_flag_eq(n, cls, c, flag, s_);
            exclusive_scan_i32(flag, pos, n, tmp, s_);
            launch_compact(n, flag, pos, list, s_);
            kernels_ += 5;
            classes.push_back({c, counts[c]});
            lists.push_back(list);
        }
        // the class lists stay allocated below `mark` while the classes run
        for (size_t i = 0; i < classes.size(); ++i) {
            const Arena::Mark cmark = arena_.mark();
            do_class(classes[i].first, lists[i], classes[i].second);
            arena_.reset(cmark);
        }
        arena_.reset(mark);
    }
    tt.stop();
    res->h_enum_ms = ms_since(h3);
    res->t_pre_ms = preprocess_ms(g_);  // (the preprocessing finished long ago; no extra wait)
    stream_sync(s_);
    res->t_enum_ms = tt.collect();
    clock_.collect(t_expand_ms_, t_count_ms_, t_root_ms_, t_setup_ms_, t_build_ms_);
    // keep answering the other shards until everyone is done
    if (o_.bound_sync) {
        int32_t gactive = 1;
        int guard = 0;
        while (gactive && guard++ < (1 << 30)) {
            int32_t gb = o_.bound_sync(best_, 0, &gactive, o_.bound_sync_user);
            if (gb < 0) fail(MCE_ERR_SYNC, "bound_sync reported a failed exchange");
            if (gb > best_) best_ = gb;
        }
    }
    res->omega = res_size_;
    res->count = res_count_;
    if (find_one_) {
        res->rows = std::move(rows_);
    } else if (stored_ > 0 && res_size_ > 0) {
        // canonical read-out on the device (canon.cu); the rows stay in the
        // result's device buffer and go straight to the caller's destination
        // in mce_result_cliques (no intermediate host copy)
        const auto h4 = clk::now();
        g_->pool.reset();
        res->device = g_->device;
        res->drows.alloc((size_t)stored_ * res_size_);
        if (canonicalize_device(g_->store.get(), stored_, res_size_, n, res->drows.get(), g_->pool, s_)) {
            int merge_passes = 0;  // CUB merge sort: block sort + (partition, merge) per doubling of tiles
            for (int64_t t = 512; t < stored_; t <<= 1) ++merge_passes;
            kernels_ += 4 + 2 * merge_passes;
            res->canonical = true;
            stream_sync(s_);
        } else {  // rows too wide: the host sorts them (mce_result_cliques)
            res->drows.release();
            res->rows.resize((size_t)stored_ * res_size_);
            MCE_CUDA(cudaMemcpyAsync(res->rows.data(), g_->store.get(), sizeof(int32_t) * stored_ * res_size_,
                                     cudaMemcpyDeviceToHost, s_));
            stream_sync(s_);
        }
        res->h_readout_ms = ms_since(h4);
    }
    res->stored = res_size_ <= 0 ? 0 : (res->drows.get() ? stored_ : (int64_t)res->rows.size() / res_size_);
    res->truncated = truncated_ ? 1 : 0;
    res->level_entries = level_entries_;
    res->t_count_ms = t_count_ms_;
    res->count_launches = count_launches_;
    res->count_bytes = count_bytes_;
    res->t_expand_ms = t_expand_ms_;
    res->t_root_ms = t_root_ms_;
    res->t_setup_ms = t_setup_ms_;
    res->t_build_ms = t_build_ms_;
    res->build_launches = build_launches_;
    if (build_launches_ > 0) {
        unsigned long long *hb = g_->host.get<unsigned long long>(1);
        MCE_CUDA(cudaMemcpyAsync(hb, build_bytes_, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s_));
        stream_sync(s_);
        res->build_bytes = (double)hb[0];
    }
    res->root_launches = root_launches_;
    res->root_bytes = root_bytes_;
    res->kernels = kernels_;
    res->h_total_ms = ms_since(h0);
    res->syncs = g_syncs - syncs0;
    return res;
}

}  // namespace

mce_result *run_engine(mce_graph *g, const mce_options &o, bool find_one) {
    Engine e(g, o, find_one);
    return e.run();
}

}  // namespace mce
