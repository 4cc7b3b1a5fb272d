/*
 * cuts_oracle.c — TEST INFRASTRUCTURE ONLY.  The plain, slow, single-threaded
 * CPU reference for cuTS subgraph-isomorphism search (Xiang et al., SC '21).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header,
 * table or helper with the CUDA path under paper_conf_sc_xiangkshs21_b200/.
 *
 * Citations "P:n" are /root/reference/PAPER.md line n.
 *
 * What it computes (plain definition; readings in DESIGN.md §2):
 *   Emb(Q, D) = { f : V_Q -> V_D injective | {u,w} in E_Q => {f(u),f(w)} in E_D }
 *   (Def. 2-4: subgraph G' with E' ⊆ E ∩ (V'×V') → non-induced,
 *   reading P1; ordered embeddings with no symmetry breaking, reading P2).
 *
 * How (the paper's algorithm, step by step, in its order):
 *   - order S: q0 = max-degree query vertex, ties → min id; each
 *     next vertex = max-degree unmatched vertex adjacent to the matched set,
 *     ties → min id (readings P5, P6).  Any valid order may be
 *     passed instead.
 *   - level 1: every data vertex u with deg(u) >= deg(q0), ascending id
 *     (Alg. 1 l.8-11), optionally restricted to positions
 *     [root_begin, root_end) of that list.
 *   - extension of a partial path to position i (Alg. 1 l.24-35):
 *     the candidates are the intersection of N(f(S[j])) over the backward
 *     neighbours j of S[i] (next_neigh), computed as the
 *     c-intersection of Alg. 2 l.19-31 with the FIRST backward
 *     neighbour's list as the initial set; a candidate c survives iff
 *     deg(c) >= deg_Q(S[i]) (degree filter, Def. 5 P:267-270, P:528-529,
 *     reading P8) and c is not already on the path (injectivity, P:211-216,
 *     reading P7).
 *   - every surviving extension is counted in level_sizes[i+1]; paths of
 *     length k are the embeddings.  Counts are exact in unsigned __int128.
 *
 * Parity pins for every function are in tests/test_oracle.py (closed forms,
 * brute force over all injective maps, networkx VF2 monomorphisms, scipy
 * traces, Fig. 3 worked trie example).  No function here is "parity unpinned".
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_OK 0
#define ORC_EINVAL (-1)
#define ORC_ENOMEM (-2)
#define ORC_EUNSUPPORTED (-7)
#define ORC_MAXK 16

typedef unsigned __int128 u128;

typedef struct {
    /* data graph D */
    uint32_t n;
    const uint64_t* row_ptr;
    const uint32_t* col;
    /* query, in matching-order positions */
    uint32_t k;
    uint32_t S[ORC_MAXK];        /* S[i] = query vertex matched at position i          */
    uint32_t qdeg[ORC_MAXK];     /* deg_Q(S[i])                                          */
    uint32_t nbw[ORC_MAXK];      /* number of backward neighbours of position i          */
    uint32_t bw[ORC_MAXK][ORC_MAXK]; /* positions j < i with (S[j], S[i]) in E_Q, ascending */
    /* state */
    uint32_t f[ORC_MAXK];        /* f[i] = data vertex matched to S[i]                  */
    u128 level[ORC_MAXK + 1];
    /* enumeration */
    uint32_t* rows;
    uint64_t cap_rows;
    u128 n_rows;
} orc_state;

static uint64_t deg(const orc_state* st, uint32_t v) {
    return st->row_ptr[v + 1] - st->row_ptr[v];
}

static int cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return (x > y) - (x < y);
}

/* membership of c in N(v): library binary search over the sorted row */
static int adjacent(const orc_state* st, uint32_t v, uint32_t c) {
    uint64_t b = st->row_ptr[v], e = st->row_ptr[v + 1];
    if (e == b) return 0;
    return bsearch(&c, st->col + b, (size_t)(e - b), sizeof(uint32_t), cmp_u32) != NULL;
}

/* ------------------------------------------------------------- validation */
int oracle_validate_graph(uint32_t n, const uint64_t* row_ptr, const uint32_t* col) {
    if (row_ptr[0] != 0) return ORC_EINVAL;
    for (uint32_t v = 0; v < n; ++v) {
        if (row_ptr[v + 1] < row_ptr[v]) return ORC_EINVAL;
        for (uint64_t p = row_ptr[v]; p < row_ptr[v + 1]; ++p) {
            uint32_t u = col[p];
            if (u >= n || u == v) return ORC_EINVAL;               /* range, self loop */
            if (p > row_ptr[v] && col[p - 1] >= u) return ORC_EINVAL; /* sorted, no dups */
        }
    }
    orc_state st;
    st.n = n; st.row_ptr = row_ptr; st.col = col;
    for (uint32_t v = 0; v < n; ++v)                                 /* symmetry */
        for (uint64_t p = row_ptr[v]; p < row_ptr[v + 1]; ++p)
            if (!adjacent(&st, col[p], v)) return ORC_EINVAL;
    return ORC_OK;
}

static int q_adj(uint32_t k, const uint32_t* qrow, const uint32_t* qcol, uint32_t a, uint32_t b) {
    (void)k;
    for (uint32_t p = qrow[a]; p < qrow[a + 1]; ++p)
        if (qcol[p] == b) return 1;
    return 0;
}

static int validate_query(uint32_t k, const uint32_t* qrow, const uint32_t* qcol) {
    if (k < 1 || k > ORC_MAXK) return ORC_EINVAL;
    if (qrow[0] != 0) return ORC_EINVAL;
    for (uint32_t a = 0; a < k; ++a) {
        if (qrow[a + 1] < qrow[a]) return ORC_EINVAL;
        for (uint32_t p = qrow[a]; p < qrow[a + 1]; ++p) {
            uint32_t b = qcol[p];
            if (b >= k || b == a) return ORC_EINVAL;
            for (uint32_t p2 = qrow[a]; p2 < p; ++p2)
                if (qcol[p2] == b) return ORC_EINVAL;
            if (!q_adj(k, qrow, qcol, b, a)) return ORC_EINVAL;
        }
    }
    /* connected (disconnected Q is handled by components; NEXT-3) */
    uint32_t seen = 1u, grown = 1;
    while (grown) {
        grown = 0;
        for (uint32_t a = 0; a < k; ++a)
            if (seen & (1u << a))
                for (uint32_t p = qrow[a]; p < qrow[a + 1]; ++p)
                    if (!(seen & (1u << qcol[p]))) { seen |= 1u << qcol[p]; grown = 1; }
    }
    if (seen != ((k == 32) ? 0xFFFFFFFFu : ((1u << k) - 1))) return ORC_EUNSUPPORTED;
    return ORC_OK;
}

/* ---------------------------------------------------------- matching order */
/* The paper's rule: root = max degree, ties min id; then the
 * max-degree vertex adjacent to the matched set, ties min id.             */
int oracle_order(uint32_t k, const uint32_t* qrow, const uint32_t* qcol, uint32_t* order) {
    int rc = validate_query(k, qrow, qcol);
    if (rc) return rc;
    uint32_t used[ORC_MAXK] = {0};
    uint32_t best = 0;
    for (uint32_t a = 1; a < k; ++a)
        if (qrow[a + 1] - qrow[a] > qrow[best + 1] - qrow[best]) best = a;
    order[0] = best; used[best] = 1;
    for (uint32_t i = 1; i < k; ++i) {
        int pick = -1;
        for (uint32_t a = 0; a < k; ++a) {
            if (used[a]) continue;
            int touches = 0;
            for (uint32_t j = 0; j < i; ++j)
                if (q_adj(k, qrow, qcol, a, order[j])) touches = 1;
            if (!touches) continue;
            if (pick < 0 || qrow[a + 1] - qrow[a] > qrow[pick + 1] - qrow[pick]) pick = (int)a;
        }
        if (pick < 0) return ORC_EUNSUPPORTED;
        order[i] = (uint32_t)pick; used[pick] = 1;
    }
    return ORC_OK;
}

static int setup(orc_state* st, uint32_t n, const uint64_t* row_ptr, const uint32_t* col,
                 uint32_t k, const uint32_t* qrow, const uint32_t* qcol, const uint32_t* order) {
    memset(st, 0, sizeof(*st));
    st->n = n; st->row_ptr = row_ptr; st->col = col; st->k = k;
    int rc = validate_query(k, qrow, qcol);
    if (rc) return rc;
    uint32_t S[ORC_MAXK];
    if (order) {
        uint32_t used[ORC_MAXK] = {0};
        for (uint32_t i = 0; i < k; ++i) {
            if (order[i] >= k || used[order[i]]) return ORC_EINVAL;
            used[order[i]] = 1;
            S[i] = order[i];
        }
    } else {
        rc = oracle_order(k, qrow, qcol, S);
        if (rc) return rc;
    }
    for (uint32_t i = 0; i < k; ++i) {
        st->S[i] = S[i];
        st->qdeg[i] = qrow[S[i] + 1] - qrow[S[i]];
        st->nbw[i] = 0;
        for (uint32_t j = 0; j < i; ++j)
            if (q_adj(k, qrow, qcol, S[j], S[i])) st->bw[i][st->nbw[i]++] = j;
        if (i > 0 && st->nbw[i] == 0) return ORC_EINVAL; /* order must stay connected */
    }
    return ORC_OK;
}

static void emit(orc_state* st) {
    if (st->rows && st->n_rows < (u128)st->cap_rows) {
        uint32_t* r = st->rows + (uint64_t)st->n_rows * st->k;
        for (uint32_t i = 0; i < st->k; ++i) r[st->S[i]] = st->f[i];  /* query-id order */
    }
    st->n_rows++;
}

/* extend the partial path f[0..i-1] by position i (Alg. 2 c-intersection) */
static void rec(orc_state* st, uint32_t i) {
    uint32_t src = st->f[st->bw[i][0]];          /* first backward neighbour (Alg. 1 l.30-31) */
    for (uint64_t p = st->row_ptr[src]; p < st->row_ptr[src + 1]; ++p) {
        uint32_t c = st->col[p];
        int ok = 1;
        for (uint32_t t = 1; t < st->nbw[i] && ok; ++t)        /* in every other list */
            ok = adjacent(st, st->f[st->bw[i][t]], c);
        if (!ok) continue;
        if (deg(st, c) < st->qdeg[i]) continue;                   /* degree filter */
        for (uint32_t j = 0; j < i && ok; ++j)                    /* injectivity */
            ok = st->f[j] != c;
        if (!ok) continue;
        st->f[i] = c;
        st->level[i + 1]++;
        if (i + 1 == st->k) emit(st);
        else rec(st, i + 1);
    }
}

static void run(orc_state* st, uint64_t root_begin, uint64_t root_end) {
    uint64_t pos = 0;   /* position in the canonical level-1 list */
    for (uint32_t v = 0; v < st->n; ++v) {
        if (deg(st, v) < st->qdeg[0]) continue;                  /* Alg. 1 l.10 */
        if (pos >= root_begin && pos < root_end) {
            st->f[0] = v;
            st->level[1]++;
            if (st->k == 1) emit(st);
            else rec(st, 1);
        }
        ++pos;
    }
}

/* Count ordered non-induced embeddings.  level_lo/level_hi (k+1 entries, may be
 * NULL): 128-bit level sizes, level[j] = partial paths with j matched vertices.
 * root range: positions [root_begin, root_end) of the canonical level-1 list.  */
int oracle_count(uint32_t n, const uint64_t* row_ptr, const uint32_t* col,
                 uint32_t k, const uint32_t* qrow, const uint32_t* qcol, const uint32_t* order,
                 uint64_t root_begin, uint64_t root_end,
                 uint64_t* count_lo, uint64_t* count_hi,
                 uint64_t* level_lo, uint64_t* level_hi) {
    orc_state* st = (orc_state*)malloc(sizeof(orc_state));
    if (!st) return ORC_ENOMEM;
    int rc = setup(st, n, row_ptr, col, k, qrow, qcol, order);
    if (rc) { free(st); return rc; }
    run(st, root_begin, root_end);
    *count_lo = (uint64_t)st->n_rows;
    *count_hi = (uint64_t)(st->n_rows >> 64);
    for (uint32_t j = 0; j <= k; ++j) {
        if (level_lo) level_lo[j] = (uint64_t)st->level[j];
        if (level_hi) level_hi[j] = (uint64_t)(st->level[j] >> 64);
    }
    free(st);
    return ORC_OK;
}

static uint32_t g_sort_k;
static int cmp_row(const void* a, const void* b) {
    const uint32_t* x = (const uint32_t*)a;
    const uint32_t* y = (const uint32_t*)b;
    for (uint32_t i = 0; i < g_sort_k; ++i)
        if (x[i] != y[i]) return x[i] < y[i] ? -1 : 1;
    return 0;
}

/* Enumerate: rows of k u32 in query-vertex-id order, sorted lexicographically
 * when all rows fit (n_found <= cap_rows).                                     */
int oracle_enumerate(uint32_t n, const uint64_t* row_ptr, const uint32_t* col,
                     uint32_t k, const uint32_t* qrow, const uint32_t* qcol, const uint32_t* order,
                     uint64_t root_begin, uint64_t root_end,
                     uint32_t* rows, uint64_t cap_rows, uint64_t* n_found) {
    orc_state* st = (orc_state*)malloc(sizeof(orc_state));
    if (!st) return ORC_ENOMEM;
    int rc = setup(st, n, row_ptr, col, k, qrow, qcol, order);
    if (rc) { free(st); return rc; }
    st->rows = rows; st->cap_rows = cap_rows;
    run(st, root_begin, root_end);
    *n_found = (uint64_t)st->n_rows;
    uint64_t nr = st->n_rows < (u128)cap_rows ? (uint64_t)st->n_rows : cap_rows;
    g_sort_k = k;
    qsort(rows, (size_t)nr, (size_t)k * sizeof(uint32_t), cmp_row);
    free(st);
    return ORC_OK;
}

/* Canonical level-1 list size (vertices with deg >= deg_Q(S[0])). */
int oracle_level1_size(uint32_t n, const uint64_t* row_ptr, uint32_t min_deg, uint64_t* out) {
    uint64_t c = 0;
    for (uint32_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] - row_ptr[v] >= min_deg) ++c;
    *out = c;
    return ORC_OK;
}

/* Decode a trie stored as per-level candidate arrays (CA) and parent arrays (PA)
 * (Fig. 3C): for every leaf of the last level, walk the parent
 * indices up to level 1 and write the root-to-leaf path (L u32 per row).
 * ca[l] has sizes[l] entries; pa[l][x] indexes level l-1 (pa[0] unused).     */
int oracle_trie_decode(uint32_t nlevels, const uint64_t* sizes,
                       const uint32_t* const* ca, const uint32_t* const* pa, uint32_t* out) {
    if (nlevels == 0) return ORC_EINVAL;
    uint32_t L = nlevels;
    for (uint64_t x = 0; x < sizes[L - 1]; ++x) {
        uint64_t at = x;
        for (int l = (int)L - 1; l >= 0; --l) {
            if (at >= sizes[l]) return ORC_EINVAL;
            out[x * L + (uint32_t)l] = ca[l][at];
            if (l > 0) at = pa[l][at];
        }
    }
    return ORC_OK;
}

/* ====================================================== directed (NEXT-1)
 * "we consider directed graphs (edges are directed)"; an undirected
 * graph is the special case with both arcs.  Plain definition (reading P1 for
 * directed graphs):
 *   Emb(Q, D) = { f injective | (u,w) in E_Q => (f(u),f(w)) in E_D }.
 * The data graph is given as out-CSR (children, D.cs) and in-CSR (parents,
 * D.ps), both sorted.  Step by step:
 *   - order: root = max out-degree ("out degree in the case of directed
 *     graphs"; reading P26), ties min id; next = max out-degree unmatched
 *     vertex weakly adjacent to the matched set (P:545 weak connectivity),
 *     ties min id.  Q must be weakly connected.
 *   - degree filter (Def. 5, with "degree (in degree and out
 *     degree)" of P:262-264; reading P27): outdeg(c) >= outdeg_Q(S[i]) and
 *     indeg(c) >= indeg_Q(S[i]).
 *   - extension of position i: for every backward neighbour j, an arc
 *     S[j] -> S[i] requires c in children(f(S[j])) (c-intersection, Alg. 2
 *     l.19-31) and an arc S[i] -> S[j] requires c in parents(f(S[j]))
 *     (p-intersection, Alg. 2 l.33-42).  The initial set is the
 *     first requirement's list (children before parents, lower j first).
 */
typedef struct {
    uint32_t n;
    const uint64_t *orow, *irow;
    const uint32_t *ocol, *icol;
    uint32_t k;
    uint32_t S[ORC_MAXK];
    uint32_t qout[ORC_MAXK], qin[ORC_MAXK];
    uint32_t nreq[ORC_MAXK];
    uint32_t req_pos[ORC_MAXK][2 * ORC_MAXK];   /* backward position j                    */
    uint32_t req_par[ORC_MAXK][2 * ORC_MAXK];   /* 0: c in children(f(S[j])), 1: parents  */
    uint32_t f[ORC_MAXK];
    u128 level[ORC_MAXK + 1];
    uint32_t* rows;
    uint64_t cap_rows;
    u128 n_rows;
} orc_di;

static int di_in_list(const uint64_t* row, const uint32_t* col, uint32_t v, uint32_t c) {
    uint64_t b = row[v], e = row[v + 1];
    if (e == b) return 0;
    return bsearch(&c, col + b, (size_t)(e - b), sizeof(uint32_t), cmp_u32) != NULL;
}

static int di_q_arc(const uint32_t* qrow, const uint32_t* qcol, uint32_t a, uint32_t b) {
    for (uint32_t p = qrow[a]; p < qrow[a + 1]; ++p)
        if (qcol[p] == b) return 1;
    return 0;
}

/* out-degree of query vertex a; in-degree by scanning every row */
static uint32_t di_q_out(const uint32_t* qrow, uint32_t a) { return qrow[a + 1] - qrow[a]; }
static uint32_t di_q_in(uint32_t k, const uint32_t* qrow, const uint32_t* qcol, uint32_t a) {
    uint32_t c = 0;
    for (uint32_t u = 0; u < k; ++u) c += (uint32_t)di_q_arc(qrow, qcol, u, a);
    return c;
}

static int di_setup(orc_di* st, uint32_t n, const uint64_t* orow, const uint32_t* ocol,
                    const uint64_t* irow, const uint32_t* icol, uint32_t k,
                    const uint32_t* qrow, const uint32_t* qcol, const uint32_t* order) {
    memset(st, 0, sizeof(*st));
    st->n = n; st->orow = orow; st->ocol = ocol; st->irow = irow; st->icol = icol; st->k = k;
    if (k < 1 || k > ORC_MAXK || qrow[0] != 0) return ORC_EINVAL;
    for (uint32_t a = 0; a < k; ++a) {
        if (qrow[a + 1] < qrow[a]) return ORC_EINVAL;
        for (uint32_t p = qrow[a]; p < qrow[a + 1]; ++p) {
            if (qcol[p] >= k || qcol[p] == a) return ORC_EINVAL;
            for (uint32_t p2 = qrow[a]; p2 < p; ++p2)
                if (qcol[p2] == qcol[p]) return ORC_EINVAL;
        }
    }
    uint32_t used[ORC_MAXK] = {0};
    if (order) {
        for (uint32_t i = 0; i < k; ++i) {
            if (order[i] >= k || used[order[i]]) return ORC_EINVAL;
            used[order[i]] = 1;
            st->S[i] = order[i];
        }
    } else {
        for (uint32_t i = 0; i < k; ++i) {
            int pick = -1;
            for (uint32_t a = 0; a < k; ++a) {
                if (used[a]) continue;
                int touches = (i == 0);
                for (uint32_t j = 0; j < i; ++j)
                    if (di_q_arc(qrow, qcol, a, st->S[j]) || di_q_arc(qrow, qcol, st->S[j], a)) touches = 1;
                if (!touches) continue;
                if (pick < 0 || di_q_out(qrow, a) > di_q_out(qrow, (uint32_t)pick)) pick = (int)a;
            }
            if (pick < 0) return ORC_EUNSUPPORTED;   /* not weakly connected */
            st->S[i] = (uint32_t)pick; used[pick] = 1;
        }
    }
    for (uint32_t i = 0; i < k; ++i) {
        uint32_t a = st->S[i];
        st->qout[i] = di_q_out(qrow, a);
        st->qin[i] = di_q_in(k, qrow, qcol, a);
        for (uint32_t j = 0; j < i; ++j)
            if (di_q_arc(qrow, qcol, st->S[j], a)) { st->req_pos[i][st->nreq[i]] = j; st->req_par[i][st->nreq[i]++] = 0; }
        for (uint32_t j = 0; j < i; ++j)
            if (di_q_arc(qrow, qcol, a, st->S[j])) { st->req_pos[i][st->nreq[i]] = j; st->req_par[i][st->nreq[i]++] = 1; }
        if (i > 0 && st->nreq[i] == 0) return order ? ORC_EINVAL : ORC_EUNSUPPORTED;
    }
    return ORC_OK;
}

static void di_emit(orc_di* st) {
    if (st->rows && st->n_rows < (u128)st->cap_rows) {
        uint32_t* r = st->rows + (uint64_t)st->n_rows * st->k;
        for (uint32_t i = 0; i < st->k; ++i) r[st->S[i]] = st->f[i];
    }
    st->n_rows++;
}

static int di_degree_ok(const orc_di* st, uint32_t c, uint32_t i) {
    return st->orow[c + 1] - st->orow[c] >= st->qout[i] && st->irow[c + 1] - st->irow[c] >= st->qin[i];
}

static void di_rec(orc_di* st, uint32_t i) {
    uint32_t v0 = st->f[st->req_pos[i][0]];
    const uint64_t* row = st->req_par[i][0] ? st->irow : st->orow;
    const uint32_t* col = st->req_par[i][0] ? st->icol : st->ocol;
    for (uint64_t p = row[v0]; p < row[v0 + 1]; ++p) {
        uint32_t c = col[p];
        int ok = 1;
        for (uint32_t t = 1; t < st->nreq[i] && ok; ++t) {
            uint32_t v = st->f[st->req_pos[i][t]];
            ok = st->req_par[i][t] ? di_in_list(st->irow, st->icol, v, c)   /* p-intersection */
                                   : di_in_list(st->orow, st->ocol, v, c);  /* c-intersection */
        }
        if (!ok || !di_degree_ok(st, c, i)) continue;
        for (uint32_t j = 0; j < i && ok; ++j) ok = st->f[j] != c;
        if (!ok) continue;
        st->f[i] = c;
        st->level[i + 1]++;
        if (i + 1 == st->k) di_emit(st);
        else di_rec(st, i + 1);
    }
}

static void di_run(orc_di* st) {
    for (uint32_t v = 0; v < st->n; ++v) {
        if (!di_degree_ok(st, v, 0)) continue;
        st->f[0] = v;
        st->level[1]++;
        if (st->k == 1) di_emit(st);
        else di_rec(st, 1);
    }
}

/* Directed count (+ level sizes, k+1 entries, may be NULL) / enumerate. */
int oracle_di_count(uint32_t n, const uint64_t* orow, const uint32_t* ocol, const uint64_t* irow,
                    const uint32_t* icol, uint32_t k, const uint32_t* qrow, const uint32_t* qcol,
                    const uint32_t* order, uint64_t* count_lo, uint64_t* count_hi,
                    uint64_t* level_lo, uint64_t* level_hi, uint32_t* rows, uint64_t cap_rows) {
    orc_di* st = (orc_di*)malloc(sizeof(orc_di));
    if (!st) return ORC_ENOMEM;
    int rc = di_setup(st, n, orow, ocol, irow, icol, k, qrow, qcol, order);
    if (rc) { free(st); return rc; }
    st->rows = rows; st->cap_rows = rows ? cap_rows : 0;
    di_run(st);
    *count_lo = (uint64_t)st->n_rows;
    *count_hi = (uint64_t)(st->n_rows >> 64);
    for (uint32_t j = 0; j <= k; ++j) {
        if (level_lo) level_lo[j] = (uint64_t)st->level[j];
        if (level_hi) level_hi[j] = (uint64_t)(st->level[j] >> 64);
    }
    if (rows) {
        uint64_t nr = st->n_rows < (u128)cap_rows ? (uint64_t)st->n_rows : cap_rows;
        g_sort_k = k;
        qsort(rows, (size_t)nr, (size_t)k * sizeof(uint32_t), cmp_row);
    }
    free(st);
    return ORC_OK;
}

int oracle_di_order(uint32_t k, const uint32_t* qrow, const uint32_t* qcol, uint32_t* order) {
    orc_di* st = (orc_di*)malloc(sizeof(orc_di));
    if (!st) return ORC_ENOMEM;
    uint64_t z[2] = {0, 0};
    int rc = di_setup(st, 0, z, NULL, z, NULL, k, qrow, qcol, NULL);
    if (!rc) memcpy(order, st->S, k * sizeof(uint32_t));
    free(st);
    return rc;
}

/* ============================================ disconnected Q
 * "If the query graph is not connected ... we split Q into a set of connected
 * components, compute sub-graph isomorphism on each of these components, and
 * produce the final result as the cross product of individual solutions."
 * Reading P16: an element of the result is still a subgraph
 * isomorphism (Def. 4), i.e. injective, so only the combinations
 * whose images are disjoint are kept.
 *
 * Step by step: the caller passes each component's embeddings (rows from
 * oracle_enumerate of the component as its own query; comp_verts[c][t] is the
 * query vertex of column t); this function walks the cross product with
 * nested loops (one level per component), keeps a combination iff no data
 * vertex repeats, counts it in 128 bits and, if `rows` is given, writes it in
 * query-id order (unsorted; the caller sorts).  Nothing is materialised
 * beyond the k-vertex partial combination.                                 */
typedef struct {
    uint32_t k, ncomp;
    const uint32_t* size;            /* vertices per component              */
    const uint32_t* const* verts;    /* query vertex ids per component      */
    const uint32_t* const* crow;     /* component rows (count x size)       */
    const uint64_t* ccount;          /* rows per component                  */
    uint32_t f[ORC_MAXK];            /* f[query vertex] (partial)           */
    uint32_t used[ORC_MAXK];         /* data vertices placed so far         */
    uint32_t nused;
    uint32_t* rows;
    uint64_t cap;
    u128 n;
} orc_cross;

static void cross_rec(orc_cross* x, uint32_t c) {
    if (c == x->ncomp) {
        if (x->rows && x->n < (u128)x->cap) memcpy(x->rows + (uint64_t)x->n * x->k, x->f, x->k * sizeof(uint32_t));
        x->n++;
        return;
    }
    const uint32_t s = x->size[c];
    for (uint64_t r = 0; r < x->ccount[c]; ++r) {
        const uint32_t* row = x->crow[c] + r * s;
        int ok = 1;
        for (uint32_t t = 0; t < s && ok; ++t)          /* injectivity across components */
            for (uint32_t u = 0; u < x->nused && ok; ++u) ok = x->used[u] != row[t];
        if (!ok) continue;
        for (uint32_t t = 0; t < s; ++t) { x->f[x->verts[c][t]] = row[t]; x->used[x->nused + t] = row[t]; }
        x->nused += s;
        cross_rec(x, c + 1);
        x->nused -= s;
    }
}

int oracle_cross_product(uint32_t k, uint32_t ncomp, const uint32_t* size, const uint32_t* const* verts,
                         const uint32_t* const* crow, const uint64_t* ccount,
                         uint32_t* rows, uint64_t cap_rows, uint64_t* count_lo, uint64_t* count_hi) {
    if (k < 1 || k > ORC_MAXK || ncomp < 1 || ncomp > k) return ORC_EINVAL;
    orc_cross x;
    memset(&x, 0, sizeof x);
    x.k = k; x.ncomp = ncomp; x.size = size; x.verts = verts; x.crow = crow; x.ccount = ccount;
    x.rows = rows; x.cap = rows ? cap_rows : 0;
    cross_rec(&x, 0);
    *count_lo = (uint64_t)x.n;
    *count_hi = (uint64_t)(x.n >> 64);
    if (rows) {
        uint64_t nr = x.n < (u128)cap_rows ? (uint64_t)x.n : cap_rows;
        g_sort_k = k;
        qsort(rows, (size_t)nr, (size_t)k * sizeof(uint32_t), cmp_row);
    }
    return ORC_OK;
}

/* ========================================= root-parallel driver (N cores)
 * SURVEY §8.c step 5 / BASELINE.md §4: level-1 roots are independent
 * sub-trees, so disjoint ranges of the canonical level-1 list
 * can be counted by separate threads with the same rec() and summed — exact
 * by construction.  Threads pull ranges of `grain` roots from an atomic
 * counter.  Used only for the CPU baseline timing (bench.py cpu_baseline);
 * every parity pin goes through the single-threaded oracle_count.           */
#include <pthread.h>

typedef struct {
    orc_state st;
    const uint32_t* canon;
    uint64_t begin, end, grain;
    uint64_t* next;                  /* shared: next root position to hand out */
} orc_worker;

static void* worker_main(void* arg) {
    orc_worker* w = (orc_worker*)arg;
    for (;;) {
        uint64_t a = __atomic_fetch_add(w->next, w->grain, __ATOMIC_RELAXED);
        if (a >= w->end) break;
        uint64_t b = a + w->grain < w->end ? a + w->grain : w->end;
        for (uint64_t p = a; p < b; ++p) {
            w->st.f[0] = w->canon[p];
            w->st.level[1]++;
            if (w->st.k == 1) emit(&w->st);
            else rec(&w->st, 1);
        }
    }
    return NULL;
}

int oracle_count_mt(uint32_t nthreads, uint32_t n, const uint64_t* row_ptr, const uint32_t* col,
                    uint32_t k, const uint32_t* qrow, const uint32_t* qcol, const uint32_t* order,
                    uint64_t root_begin, uint64_t root_end, uint64_t grain,
                    uint64_t* count_lo, uint64_t* count_hi) {
    if (nthreads < 1 || nthreads > 1024 || grain < 1) return ORC_EINVAL;
    orc_worker* w = (orc_worker*)calloc(nthreads, sizeof(orc_worker));
    pthread_t* th = (pthread_t*)calloc(nthreads, sizeof(pthread_t));
    uint32_t* canon = (uint32_t*)malloc(((size_t)n + 1) * sizeof(uint32_t));
    if (!w || !th || !canon) { free(w); free(th); free(canon); return ORC_ENOMEM; }
    int rc = setup(&w[0].st, n, row_ptr, col, k, qrow, qcol, order);
    if (rc) { free(w); free(th); free(canon); return rc; }
    uint64_t nc = 0;                                    /* canonical level-1 list (Alg. 1 l.8-11) */
    for (uint32_t v = 0; v < n; ++v)
        if (deg(&w[0].st, v) >= w[0].st.qdeg[0]) canon[nc++] = v;
    uint64_t b = root_begin < nc ? root_begin : nc, e = root_end < nc ? root_end : nc;
    if (e < b) e = b;
    uint64_t next = b;
    for (uint32_t t = 0; t < nthreads; ++t) {
        if (t) w[t].st = w[0].st;
        w[t].canon = canon; w[t].begin = b; w[t].end = e; w[t].grain = grain; w[t].next = &next;
    }
    uint32_t started = 0;
    for (; started < nthreads; ++started)
        if (pthread_create(&th[started], NULL, worker_main, &w[started]) != 0) break;
    if (started == 0) worker_main(&w[0]);
    for (uint32_t t = 0; t < started; ++t) pthread_join(th[t], NULL);
    u128 tot = 0;
    for (uint32_t t = 0; t < nthreads; ++t) tot += w[t].st.n_rows;
    *count_lo = (uint64_t)tot;
    *count_hi = (uint64_t)(tot >> 64);
    free(w); free(th); free(canon);
    return ORC_OK;
}
