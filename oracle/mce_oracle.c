/*
 * mce_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded CPU reference for the maximum-clique hot path
 * of Geil, Porumbescu & Owens, "Maximum Clique Enumeration on the GPU"
 * (IPDPS 2023; /root/reference/PAPER.md).  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference leg may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_geilpo23_b200/csrc); neither includes the other.
 *
 * Graph input everywhere: undirected simple graph as CSR with both edge
 * directions stored and every adjacency list sorted ascending by vertex id:
 *   rowptr[n+1] (int64), col[rowptr[n]] (int32).
 *
 * Functions and the passages they follow:
 *   oracle_core_numbers  -- k-core numbers (PAPER.md II-B-2, line 61: "The
 *                           largest value of k for which a vertex is a member of
 *                           a k-core is its core number"), computed with the
 *                           textbook Batagelj-Zaversnik bucket peel.
 *   oracle_greedy        -- the greedy heuristic (PAPER.md IV-A-1/IV-A-2, lines
 *                           105-109, Algorithm 1): h runs, seeds = the h
 *                           vertices with highest threshold, each run adds the
 *                           remaining candidate with the highest threshold and
 *                           filters the candidates to its neighbours.
 *   oracle_mce           -- all maximum cliques (PAPER.md II, line 47: omega(G)
 *                           and "the members of all cliques of size omega") by
 *                           the basic branching algorithm of II-A (lines 51-53)
 *                           with the |C|+|P| bound or the colouring bound of
 *                           II-B-3 (line 63).
 *   oracle_kclique_counts-- number of k-cliques for every k (the size of every
 *                           level of the unpruned breadth-first search tree,
 *                           II-D line 77: "we need to store all k-cliques at each
 *                           level of the tree").
 *   oracle_is_clique     -- definition check (II, line 47).
 *
 * Pins (tests/test_oracle.py): brute-force subset enumeration for n <= 20,
 * closed forms (K_n, C_n, Turan T(n,k), Paley P(q)), planted cliques,
 * the definition of core numbers by repeated removal, a hand-traced greedy
 * example (tests/golden/greedy_trace.txt).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* k-core numbers: Batagelj & Zaversnik, "An O(m) Algorithm for Cores         */
/* Decomposition of Networks" (2003).  Returns the degeneracy (max core).     */
/* order_out (optional): the peel order (vertex removed i-th).               */
/* ------------------------------------------------------------------------ */
int32_t oracle_core_numbers(int64_t n, const int64_t *rowptr, const int32_t *col,
                            int32_t *core, int32_t *order_out) {
    if (n == 0) return 0;
    int64_t maxdeg = 0;
    int64_t *deg = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t v = 0; v < n; ++v) {
        deg[v] = rowptr[v + 1] - rowptr[v];
        if (deg[v] > maxdeg) maxdeg = deg[v];
    }
    int64_t *bin = (int64_t *)calloc(maxdeg + 1, sizeof(int64_t));
    int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * n);
    int64_t *vert = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t v = 0; v < n; ++v) bin[deg[v]]++;
    int64_t start = 0;
    for (int64_t d = 0; d <= maxdeg; ++d) {
        int64_t num = bin[d];
        bin[d] = start;
        start += num;
    }
    for (int64_t v = 0; v < n; ++v) {
        pos[v] = bin[deg[v]];
        vert[pos[v]] = v;
        bin[deg[v]]++;
    }
    for (int64_t d = maxdeg; d >= 1; --d) bin[d] = bin[d - 1];
    bin[0] = 0;
    for (int64_t i = 0; i < n; ++i) {
        int64_t v = vert[i];
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) {
            int64_t u = col[e];
            if (deg[u] > deg[v]) {
                int64_t du = deg[u];
                int64_t pu = pos[u];
                int64_t pw = bin[du];
                int64_t w = vert[pw];
                if (u != w) {
                    pos[u] = pw;
                    vert[pu] = w;
                    pos[w] = pu;
                    vert[pw] = u;
                }
                bin[du]++;
                deg[u]--;
            }
        }
    }
    int32_t degeneracy = 0;
    for (int64_t v = 0; v < n; ++v) {
        core[v] = (int32_t)deg[v];
        if (core[v] > degeneracy) degeneracy = core[v];
    }
    if (order_out)
        for (int64_t i = 0; i < n; ++i) order_out[i] = (int32_t)vert[i];
    free(deg);
    free(bin);
    free(pos);
    free(vert);
    return degeneracy;
}

/* ------------------------------------------------------------------------ */
static int has_edge(const int64_t *rowptr, const int32_t *col, int32_t u, int32_t w) {
    int64_t lo = rowptr[u], hi = rowptr[u + 1];
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (col[mid] < w)
            lo = mid + 1;
        else
            hi = mid;
    }
    return lo < rowptr[u + 1] && col[lo] == w;
}

int32_t oracle_is_clique(const int64_t *rowptr, const int32_t *col, const int32_t *verts, int32_t k) {
    for (int32_t i = 0; i < k; ++i)
        for (int32_t j = i + 1; j < k; ++j)
            if (!has_edge(rowptr, col, verts[i], verts[j])) return 0;
    return 1;
}

/* ------------------------------------------------------------------------ */
/* Greedy heuristic, PAPER.md IV-A (lines 103-109) and Algorithm 1.          */
/*  threshold[v]: the vertex's degree or core number (IV-A: "an option to use */
/*  either the vertex degrees or core numbers for determining the greedy     */
/*  ordering").  Seeds: the h vertices with highest threshold (ties: smaller */
/*  id first).  A run starts with C = {seed}, P = N(seed); while P is not    */
/*  empty it adds the candidate with the highest threshold (ties: smaller    */
/*  id, the first maximum of a segment sorted by id -- the CUBSEGMENTEDMAX   */
/*  of Algorithm 1 line 34) and keeps only candidates adjacent to it.        */
/*  Returns the best clique size over all runs (omega-bar, Algorithm 1 line  */
/*  44).  run_size (optional, length h): size of each run, in seed order.    */
/*  best_clique (optional, capacity >= returned size): clique of the first   */
/*  run that reaches the best size, vertices in the order added.             */
/* ------------------------------------------------------------------------ */
static const int64_t *g_sort_key;
static int cmp_seed(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    if (g_sort_key[x] != g_sort_key[y]) return g_sort_key[x] > g_sort_key[y] ? -1 : 1;
    return (x > y) - (x < y);
}

int32_t oracle_greedy(int64_t n, const int64_t *rowptr, const int32_t *col, const int64_t *threshold,
                      int64_t h, int32_t *run_size, int32_t *best_clique) {
    if (n == 0 || h <= 0) return 0;
    if (h > n) h = n;
    int32_t *seeds = (int32_t *)malloc(sizeof(int32_t) * n);
    for (int64_t v = 0; v < n; ++v) seeds[v] = (int32_t)v;
    g_sort_key = threshold;
    qsort(seeds, (size_t)n, sizeof(int32_t), cmp_seed);
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < n; ++v)
        if (rowptr[v + 1] - rowptr[v] > maxdeg) maxdeg = rowptr[v + 1] - rowptr[v];
    int32_t *P = (int32_t *)malloc(sizeof(int32_t) * (maxdeg + 1));
    int32_t *C = (int32_t *)malloc(sizeof(int32_t) * (maxdeg + 2));
    int32_t best = 0;
    for (int64_t r = 0; r < h; ++r) {
        int32_t s = seeds[r];
        int32_t csize = 0;
        C[csize++] = s;
        int64_t np = 0;
        for (int64_t e = rowptr[s]; e < rowptr[s + 1]; ++e) P[np++] = col[e];
        while (np > 0) {
            int64_t bi = 0;
            for (int64_t i = 1; i < np; ++i) {
                if (threshold[P[i]] > threshold[P[bi]] ||
                    (threshold[P[i]] == threshold[P[bi]] && P[i] < P[bi]))
                    bi = i;
            }
            int32_t w = P[bi];
            C[csize++] = w;
            int64_t k = 0;
            for (int64_t i = 0; i < np; ++i)
                if (P[i] != w && has_edge(rowptr, col, w, P[i])) P[k++] = P[i];
            np = k;
        }
        if (run_size) run_size[r] = csize;
        if (csize > best) {
            best = csize;
            if (best_clique) memcpy(best_clique, C, sizeof(int32_t) * csize);
        }
    }
    free(seeds);
    free(P);
    free(C);
    return best;
}

/* ------------------------------------------------------------------------ */
/* All maximum cliques, PAPER.md II-A (lines 51-53): "begin with an empty     */
/* clique set, C, and a set of candidate vertices, P ... select a vertex      */
/* v in P to add to C, and filter out vertices in P not connected to v ...   */
/* until P is empty, then note this clique and its size. Backtrack ...".     */
/*                                                                            */
/* Visiting every clique exactly once: vertices are taken in a fixed order   */
/* pi (the Batagelj-Zaversnik peel order, so |P| <= degeneracy at the root); */
/* the root v starts with P = its neighbours later in pi, and a branch on w  */
/* keeps only the candidates not yet branched on.                            */
/*                                                                            */
/* Bounds (II-B-3, line 63): a branch is cut when its upper bound is below   */
/* the best size found so far (strict, so every clique of the maximum size   */
/* is kept -- II line 47 "all cliques of size omega"):                        */
/*   bound = 0: |C| + |P|                  ("the most straightforward")      */
/*   bound = 1: |C| + (colours of a greedy sequential colouring of P)        */
/*              ("a tighter upper bound using ... vertex coloring"; the       */
/*              colouring is Tomita & Seki's MCQ order: colour classes built */
/*              one at a time taking the lowest-index uncoloured vertex not  */
/*              adjacent to the class, branch from the highest colour down). */
/* Both give the same answer; bound=1 is the only one that terminates on the */
/* near-complete hub cores of R-MAT graphs.                                  */
/* The candidate sets of one root live in a local bitset space: local index  */
/* i <-> i-th later neighbour of the root, adjacency from the oriented lists. */
/* Results: omega, count, every maximum clique with its vertices ascending,  */
/* the cliques in lexicographic order.                                       */
/* ------------------------------------------------------------------------ */
typedef struct {
    int32_t best;
    int32_t W;         /* words per local bitset */
    int32_t bound;     /* 0 = |C|+|P|, 1 = colouring */
    const uint64_t *A; /* local adjacency, L rows of W words */
    const int32_t *V;  /* local index -> vertex id */
    int32_t *stack;    /* current clique C (vertex ids) */
    uint64_t *pool;    /* candidate bitsets, one per depth */
    int32_t *ord;      /* colouring scratch, per depth: L entries */
    int32_t *colr;
    uint64_t *scratch; /* 2 W words */
    int32_t L;
    int32_t *out;      /* found cliques of size best, flat */
    int64_t out_count;
    int64_t out_cap;
    int32_t count_only; /* 1: count the cliques of size best, store none */
    int32_t tight;      /* 1: apply the tight-node rule (see expand) */
} mce_ctx;

static void record(mce_ctx *x, int32_t size) {
    if (size > x->best) {
        x->best = size;
        x->out_count = 0;
    }
    if (x->count_only) {
        x->out_count++;
        return;
    }
    if ((x->out_count + 1) * (int64_t)size > x->out_cap) {
        int64_t cap = x->out_cap ? x->out_cap * 2 : 1024;
        while ((x->out_count + 1) * (int64_t)size > cap) cap *= 2;
        x->out = (int32_t *)realloc(x->out, sizeof(int32_t) * cap);
        x->out_cap = cap;
    }
    memcpy(x->out + x->out_count * size, x->stack, sizeof(int32_t) * size);
    x->out_count++;
}

static int32_t popcount_set(const uint64_t *s, int32_t W) {
    int32_t c = 0;
    for (int32_t i = 0; i < W; ++i) c += __builtin_popcountll(s[i]);
    return c;
}

/* C has csize vertices (x->stack[0..csize-1]); P = x->pool + csize*W. */
static void expand(mce_ctx *x, int32_t csize) {
    const int32_t W = x->W;
    uint64_t *P = x->pool + (int64_t)csize * W;
    uint64_t *Q = P + W; /* child candidates */
    int32_t *ord = x->ord + (int64_t)csize * x->L;
    int32_t *colr = x->colr + (int64_t)csize * x->L;
    int32_t np = 0;
    if (x->tight && popcount_set(P, W) + csize == x->best) {
        /* Tight node (a direct consequence of the |C|+|P| bound, II-B-3 line
         * 63): every clique below (C, P) is C + S with S a clique inside P, so
         * the only one that can have the size sought, |C| + |P|, is C + P
         * itself -- a maximum clique iff P is a clique.  Checked pair by pair
         * instead of expanding the |P| levels of single-child branches. */
        int32_t k = csize;
        for (int32_t w = 0; w < W; ++w) {
            uint64_t b = P[w];
            while (b) {
                int32_t v = w * 64 + __builtin_ctzll(b);
                b &= b - 1;
                for (int32_t j = 0; j < W; ++j) {
                    uint64_t miss = P[j] & ~x->A[(int64_t)v * W + j];
                    if (j == (v >> 6)) miss &= ~(1ULL << (v & 63));
                    if (miss) return; /* P is not a clique: nothing of size best here */
                }
                x->stack[k++] = x->V[x->L - 1 - v];
            }
        }
        record(x, k);
        return;
    }
    if (x->bound == 1) { /* greedy sequential colouring of P */
        uint64_t *U = x->scratch, *S = x->scratch + W;
        memcpy(U, P, sizeof(uint64_t) * W);
        int32_t c = 0;
        while (popcount_set(U, W)) {
            ++c;
            memcpy(S, U, sizeof(uint64_t) * W);
            for (int32_t w = 0; w < W; ++w) {
                while (S[w]) {
                    int32_t v = w * 64 + __builtin_ctzll(S[w]);
                    for (int32_t j = 0; j < W; ++j) S[j] &= ~x->A[(int64_t)v * W + j];
                    S[w] &= ~(1ULL << (v & 63));
                    U[w] &= ~(1ULL << (v & 63));
                    ord[np] = v;
                    colr[np] = c;
                    ++np;
                }
            }
        }
    } else { /* no colouring: bound |C| + (number of candidates left) */
        for (int32_t w = 0; w < W; ++w) {
            uint64_t b = P[w];
            while (b) {
                int32_t v = w * 64 + __builtin_ctzll(b);
                b &= b - 1;
                ord[np] = v;
                colr[np] = np + 1; /* candidates left when branching on ord[np] */
                ++np;
            }
        }
    }
    for (int32_t i = np - 1; i >= 0; --i) {
        if (csize + colr[i] < x->best) return;
        int32_t v = ord[i];
        x->stack[csize] = x->V[x->L - 1 - v]; /* local index v <-> V[L-1-v] (see oracle_mce) */
        int32_t nonempty = 0;
        for (int32_t j = 0; j < W; ++j) {
            Q[j] = P[j] & x->A[(int64_t)v * W + j];
            nonempty |= Q[j] != 0;
        }
        if (!nonempty) {
            if (csize + 1 >= x->best) record(x, csize + 1);
        } else {
            expand(x, csize + 1);
        }
        P[v >> 6] &= ~(1ULL << (v & 63));
    }
}

static int32_t g_k;
static int cmp_clique(const void *a, const void *b) {
    const int32_t *x = (const int32_t *)a, *y = (const int32_t *)b;
    for (int32_t i = 0; i < g_k; ++i)
        if (x[i] != y[i]) return (x[i] > y[i]) - (x[i] < y[i]);
    return 0;
}
static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

static int32_t *g_res = NULL;
static int64_t g_res_count = 0;
static int32_t g_res_omega = 0;

/* Returns the number of maximum cliques; *omega_out = clique number.
 * lb: initial lower bound (0 = none).  bound: 0 = |C|+|P|, 1 = colouring.
 * flags bit 0 (count_only): count the maximum cliques without storing them
 * (graphs whose multiplicity does not fit in memory, e.g. R-MAT scale 22);
 * bit 1 (tight): apply the tight-node rule of expand() (same answer, fewer
 * levels on long single-child chains).
 * The cliques are kept until oracle_mce_fetch() copies them out.
 * Returns -1 if some root has more than 65536 later neighbours. */
int64_t oracle_mce_ex(int64_t n, const int64_t *rowptr, const int32_t *col, int32_t lb, int32_t bound,
                      int32_t flags, int32_t *omega_out) {
    const int32_t count_only = flags & 1, tight = (flags >> 1) & 1;
    free(g_res);
    g_res = NULL;
    g_res_count = 0;
    g_res_omega = 0;
    if (n == 0) { /* the empty clique is the only clique of the null graph */
        *omega_out = 0;
        g_res_count = 1;
        return 1;
    }
    int32_t *core = (int32_t *)malloc(sizeof(int32_t) * n);
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * n);
    int32_t *pos = (int32_t *)malloc(sizeof(int32_t) * n);
    int32_t *loc = (int32_t *)malloc(sizeof(int32_t) * n);
    oracle_core_numbers(n, rowptr, col, core, order);
    for (int64_t i = 0; i < n; ++i) pos[order[i]] = (int32_t)i;
    for (int64_t i = 0; i < n; ++i) loc[i] = -1;
    /* oriented lists: later neighbours in pi, kept in pi order */
    int64_t *orp = (int64_t *)calloc(n + 1, sizeof(int64_t));
    for (int64_t v = 0; v < n; ++v)
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e)
            if (pos[col[e]] > pos[v]) orp[v + 1]++;
    for (int64_t v = 0; v < n; ++v) orp[v + 1] += orp[v];
    int32_t *ocol = (int32_t *)malloc(sizeof(int32_t) * (orp[n] + 1));
    int64_t maxout = 0;
    {
        int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * n);
        for (int64_t v = 0; v < n; ++v) fill[v] = orp[v];
        for (int64_t i = 0; i < n; ++i) { /* visiting heads w in pi order keeps every list in pi order */
            int32_t w = order[i];
            for (int64_t e = rowptr[w]; e < rowptr[w + 1]; ++e) {
                int32_t v = col[e];
                if (pos[w] > pos[v]) ocol[fill[v]++] = w;
            }
        }
        free(fill);
    }
    for (int64_t v = 0; v < n; ++v)
        if (orp[v + 1] - orp[v] > maxout) maxout = orp[v + 1] - orp[v];
    if (maxout > 65536) {
        free(core); free(order); free(pos); free(loc); free(orp); free(ocol);
        return -1;
    }
    int32_t Wmax = (int32_t)((maxout + 63) / 64);
    if (Wmax < 1) Wmax = 1;
    mce_ctx x;
    memset(&x, 0, sizeof(x));
    x.best = lb > 1 ? lb : 1;
    x.bound = bound;
    x.count_only = count_only;
    x.tight = tight;
    uint64_t *A = (uint64_t *)malloc(sizeof(uint64_t) * (maxout + 1) * Wmax);
    x.stack = (int32_t *)malloc(sizeof(int32_t) * (maxout + 2));
    x.pool = (uint64_t *)malloc(sizeof(uint64_t) * (maxout + 3) * Wmax);
    x.ord = (int32_t *)malloc(sizeof(int32_t) * (maxout + 2) * (maxout + 1));
    x.colr = (int32_t *)malloc(sizeof(int32_t) * (maxout + 2) * (maxout + 1));
    x.scratch = (uint64_t *)malloc(sizeof(uint64_t) * 2 * Wmax);
    for (int64_t i = 0; i < n; ++i) {
        int32_t r = order[i];
        int32_t L = (int32_t)(orp[r + 1] - orp[r]);
        if (1 + L < x.best) continue;
        x.stack[0] = r;
        if (L == 0) {
            record(&x, 1);
            continue;
        }
        const int32_t *V = ocol + orp[r];
        int32_t W = (L + 63) / 64;
        /* Local index of V[a] is L-1-a: bits run in reverse pi order, so the
         * greedy colouring meets the high-core vertices first and gives them the
         * low colours, and the search branches on them last, with the smallest
         * candidate sets (smallest-last order, reading 5).  The set of
         * maximum cliques found does not depend on this order, only the run time. */
        for (int32_t a = 0; a < L; ++a) loc[V[a]] = L - 1 - a;
        memset(A, 0, sizeof(uint64_t) * L * W);
        for (int32_t a = 0; a < L; ++a) {
            int32_t u = V[a];
            for (int64_t e = orp[u]; e < orp[u + 1]; ++e) {
                int32_t b = loc[ocol[e]], la = L - 1 - a;
                if (b >= 0) {
                    A[(int64_t)la * W + (b >> 6)] |= 1ULL << (b & 63);
                    A[(int64_t)b * W + (la >> 6)] |= 1ULL << (la & 63);
                }
            }
        }
        for (int32_t a = 0; a < L; ++a) loc[V[a]] = -1;
        x.W = W;
        x.L = L;
        x.A = A;
        x.V = V;
        uint64_t *P = x.pool + W; /* depth 1 */
        for (int32_t j = 0; j < W; ++j) P[j] = 0;
        for (int32_t a = 0; a < L; ++a) P[a >> 6] |= 1ULL << (a & 63);
        expand(&x, 1);
    }
    int32_t k = x.best;
    if (x.out_count == 0) k = 0; /* lb was above omega: nothing of size >= lb */
    if (count_only) {
        *omega_out = k;
        g_res_count = x.out_count;
        g_res_omega = k;
        free(A); free(x.stack); free(x.pool); free(x.ord); free(x.colr); free(x.scratch);
        free(core); free(order); free(pos); free(loc); free(orp); free(ocol);
        return g_res_count;
    }
    for (int64_t c = 0; c < x.out_count; ++c) qsort(x.out + c * k, (size_t)k, sizeof(int32_t), cmp_i32);
    g_k = k;
    if (k > 0) qsort(x.out, (size_t)x.out_count, sizeof(int32_t) * k, cmp_clique);
    g_res = x.out;
    g_res_count = x.out_count;
    g_res_omega = k;
    *omega_out = k;
    free(A); free(x.stack); free(x.pool); free(x.ord); free(x.colr); free(x.scratch);
    free(core); free(order); free(pos); free(loc); free(orp); free(ocol);
    return g_res_count;
}

int64_t oracle_mce(int64_t n, const int64_t *rowptr, const int32_t *col, int32_t lb, int32_t bound,
                   int32_t *omega_out) {
    return oracle_mce_ex(n, rowptr, col, lb, bound, 0, omega_out);
}

/* Copy the cliques of the last oracle_mce() call (count * omega int32). */
void oracle_mce_fetch(int32_t *dst) {
    if (dst && g_res && g_res_count && g_res_omega)
        memcpy(dst, g_res, sizeof(int32_t) * g_res_count * g_res_omega);
    free(g_res);
    g_res = NULL;
    g_res_count = 0;
}

/* ------------------------------------------------------------------------ */
/* Number of k-cliques for k = 1..kmax (counts[k-1]).  Each clique is counted */
/* once from its smallest vertex, extending with larger common neighbours.  */
/* Returns the largest k with a nonzero count (= omega when kmax >= omega).  */
/* ------------------------------------------------------------------------ */
static void count_rec(const int64_t *rowptr, const int32_t *col, int32_t depth, const int32_t *P,
                      int64_t np, int32_t kmax, int64_t *counts, int32_t **bufs) {
    /* every element of P completes a (depth+1)-clique */
    if (depth + 1 <= kmax) counts[depth] += np;
    if (depth + 1 >= kmax) return;
    for (int64_t i = 0; i < np; ++i) {
        int32_t w = P[i];
        int32_t *Q = bufs[depth + 1];
        int64_t nq = 0;
        for (int64_t j = i + 1; j < np; ++j)
            if (has_edge(rowptr, col, w, P[j])) Q[nq++] = P[j];
        if (nq) count_rec(rowptr, col, depth + 1, Q, nq, kmax, counts, bufs);
    }
}

int32_t oracle_kclique_counts(int64_t n, const int64_t *rowptr, const int32_t *col, int32_t kmax,
                              int64_t *counts) {
    for (int32_t k = 0; k < kmax; ++k) counts[k] = 0;
    if (n == 0 || kmax <= 0) return 0;
    counts[0] = n;
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < n; ++v)
        if (rowptr[v + 1] - rowptr[v] > maxdeg) maxdeg = rowptr[v + 1] - rowptr[v];
    int32_t **bufs = (int32_t **)malloc(sizeof(int32_t *) * (kmax + 2));
    for (int32_t d = 0; d < kmax + 2; ++d) bufs[d] = (int32_t *)malloc(sizeof(int32_t) * (maxdeg + 1));
    for (int64_t v = 0; v < n && kmax >= 2; ++v) {
        int32_t *P = bufs[1];
        int64_t np = 0;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e)
            if (col[e] > v) P[np++] = col[e];
        if (np) count_rec(rowptr, col, 1, P, np, kmax, counts, bufs);
    }
    for (int32_t d = 0; d < kmax + 2; ++d) free(bufs[d]);
    free(bufs);
    int32_t top = 0;
    for (int32_t k = 0; k < kmax; ++k)
        if (counts[k]) top = k + 1;
    return top;
}

/* ------------------------------------------------------------------------ */
/* oracle_mce_plain -- the SAME problem (PAPER.md II line 47: omega and all   */
/* cliques of size omega) by the most literal form of the basic branching    */
/* algorithm of II-A (lines 51-53) with the "most straightforward" bound of  */
/* II-B-3 (line 63: "the size of C plus the size of P").  It is written to   */
/* share nothing with oracle_mce above, nor with the CUDA path: no k-core,   */
/* no orientation by rank, no bitsets, no local index space, no colouring.   */
/*                                                                            */
/* A vertex order "<" is fixed first: plain vertex id (order = 0), or the    */
/* paper's own orientation of IV-C (line 131: "keep the edge where the       */
/* source vertex has lower degree"; order = 1: by (degree, id)).             */
/*   for every vertex v in that order:  C = {v},  P = {u in N(v) : u > v}     */
/*   EXPAND(C, P): for the i-th vertex w of P (ascending id):                 */
/*       if |C| + (|P| - i) < best: stop  (C + the vertices of P from w on    */
/*                                         cannot reach best)                 */
/*       Q = {u in P : u > w, u adjacent to w}   (list in "<" order, edge     */
/*                                 test by binary search in w's CSR row)     */
/*       Q empty  -> C + w is a clique no later vertex extends: note it       */
/*       else     -> EXPAND(C + w, Q)                                         */
/*                                                                            */
/* Every clique K = {k1 < ... < kt} is visited exactly once (root k1, then   */
/* k2, ...), and a maximum clique is always a leaf, so the cliques noted at   */
/* the final best size are exactly the maximum cliques.  Pruning is strict   */
/* (<), so cliques of size equal to best survive.                            */
/* count_only = 1 counts instead of storing.  Results are read back with     */
/* oracle_mce_fetch (same canonical order as oracle_mce).                    */
/* ------------------------------------------------------------------------ */
typedef struct {
    const int64_t *rowptr;
    const int32_t *col;
    int32_t best;
    int32_t count_only;
    int32_t *C;         /* current clique, vertex ids */
    int32_t **lists;    /* one candidate list per depth */
    int32_t *out;
    int64_t out_count;
    int64_t out_cap;
} plain_ctx;

static void plain_note(plain_ctx *x, int32_t size) {
    if (size < x->best) return;
    if (size > x->best) {
        x->best = size;
        x->out_count = 0;
    }
    if (!x->count_only) {
        if ((x->out_count + 1) * (int64_t)size > x->out_cap) {
            int64_t cap = x->out_cap ? x->out_cap * 2 : 1024;
            while ((x->out_count + 1) * (int64_t)size > cap) cap *= 2;
            x->out = (int32_t *)realloc(x->out, sizeof(int32_t) * cap);
            x->out_cap = cap;
        }
        memcpy(x->out + x->out_count * size, x->C, sizeof(int32_t) * size);
    }
    x->out_count++;
}

static void plain_expand(plain_ctx *x, int32_t csize, const int32_t *P, int64_t np) {
    int32_t *Q = x->lists[csize + 1];
    for (int64_t i = 0; i < np; ++i) {
        if (csize + (np - i) < x->best) return;
        int32_t w = P[i];
        x->C[csize] = w;
        int64_t nq = 0;
        for (int64_t j = i + 1; j < np; ++j)
            if (has_edge(x->rowptr, x->col, w, P[j])) Q[nq++] = P[j];
        if (nq == 0)
            plain_note(x, csize + 1);
        else
            plain_expand(x, csize + 1, Q, nq);
    }
}

static const int64_t *g_rank;
static int cmp_by_rank(const void *a, const void *b) {
    int64_t x = g_rank[*(const int32_t *)a], y = g_rank[*(const int32_t *)b];
    return (x > y) - (x < y);
}

int64_t oracle_mce_plain(int64_t n, const int64_t *rowptr, const int32_t *col, int32_t lb,
                         int32_t order, int32_t count_only, int32_t *omega_out) {
    free(g_res);
    g_res = NULL;
    g_res_count = 0;
    g_res_omega = 0;
    if (n == 0) { /* the empty clique is the only clique of the null graph */
        *omega_out = 0;
        g_res_count = 1;
        return 1;
    }
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < n; ++v)
        if (rowptr[v + 1] - rowptr[v] > maxdeg) maxdeg = rowptr[v + 1] - rowptr[v];
    plain_ctx x;
    memset(&x, 0, sizeof(x));
    x.rowptr = rowptr;
    x.col = col;
    x.best = lb > 1 ? lb : 1;
    x.count_only = count_only;
    /* rank[v] = position of v in the order "<": key (degree, id) or id */
    int64_t *rank = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t v = 0; v < n; ++v) rank[v] = order == 1 ? (rowptr[v + 1] - rowptr[v]) * n + v : v;
    x.C = (int32_t *)malloc(sizeof(int32_t) * (maxdeg + 2));
    x.lists = (int32_t **)malloc(sizeof(int32_t *) * (maxdeg + 3));
    for (int64_t d = 0; d < maxdeg + 3; ++d) x.lists[d] = NULL;
    for (int64_t v = 0; v < n; ++v) {
        int64_t np = 0;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) np += rank[col[e]] > rank[v];
        if (1 + np < x.best) continue;
        x.C[0] = (int32_t)v;
        if (np == 0) {
            plain_note(&x, 1);
            continue;
        }
        /* lists are allocated lazily, one per depth, each of the root's size */
        for (int64_t d = 1; d <= np + 1; ++d)
            if (!x.lists[d]) x.lists[d] = (int32_t *)malloc(sizeof(int32_t) * (maxdeg + 1));
        int32_t *P = x.lists[1];
        np = 0;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e)
            if (rank[col[e]] > rank[v]) P[np++] = col[e];
        g_rank = rank;
        qsort(P, (size_t)np, sizeof(int32_t), cmp_by_rank);
        plain_expand(&x, 1, P, np);
    }
    int32_t k = x.best;
    if (x.out_count == 0) k = 0;
    if (!count_only) {
        for (int64_t c = 0; c < x.out_count; ++c) qsort(x.out + c * k, (size_t)k, sizeof(int32_t), cmp_i32);
        g_k = k;
        if (k > 0) qsort(x.out, (size_t)x.out_count, sizeof(int32_t) * k, cmp_clique);
        g_res = x.out;
    } else {
        free(x.out);
    }
    g_res_count = x.out_count;
    g_res_omega = k;
    *omega_out = k;
    for (int64_t d = 0; d < maxdeg + 3; ++d) free(x.lists[d]);
    free(x.lists);
    free(x.C);
    free(rank);
    return g_res_count;
}
