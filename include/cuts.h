/*
 * cuts.h — C ABI of libcuts.so, the B200 (sm_100a) hot path of cuTS
 * subgraph-isomorphism search (Xiang, Khan, Serra, Halappanavar,
 * Sukumaran-Rajam, SC '21).  "P:n" cites /root/reference/PAPER.md line n.
 *
 * The library counts or enumerates the ORDERED, NON-INDUCED embeddings of a
 * small query graph Q (k <= 8 vertices) in a large undirected data
 * graph D (Def. 2-4; readings P1/P2 in DESIGN.md):
 *     Emb(Q, D) = { f : V_Q -> V_D injective | {u,w} in E_Q => {f(u),f(w)} in E_D }.
 * It does so the paper's way: level-synchronous extension of partial paths
 * stored in a trie of (parent index, data vertex) levels (Fig. 3C),
 * each extension being an intersection of backward-neighbour CSR lists
 * (Alg. 1, Alg. 2 c-intersection P:1019-1031) filtered by
 * degree (Def. 5) and injectivity, with hybrid BFS/DFS
 * chunking when a level would not fit.
 *
 * Conventions
 *   - Every call returns cuts_status; no C++ exception crosses the ABI.
 *     cuts_last_error(ctx) describes the last failing call on ctx.
 *   - Call order: create -> load_graph -> set_query -> count/enumerate.
 *     Anything else returns CUTS_ESTATE.
 *   - Ownership: the CALLER owns every large device buffer (graph, arena,
 *     enumeration output); the library borrows them and never cudaMallocs.
 *     Small host arrays (query, order) are copied.
 *   - Threading: one ctx per host thread.  Work is enqueued on opts.stream and
 *     every call is host-synchronous (returns when its result is ready).
 *   - The CUDA path is the only path: there is no CPU fallback.
 */
#ifndef CUTS_H
#define CUTS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CUTS_MAX_K 8
#define CUTS_ABI_VERSION 3

typedef struct cuts_ctx cuts_ctx;

typedef enum {
    CUTS_OK = 0,
    CUTS_EINVAL = -1,       /* bad argument, invalid graph/query/order                  */
    CUTS_ENOMEM = -2,       /* arena too small (BFS: a level does not fit) */
    CUTS_ECUDA = -3,        /* a CUDA runtime call failed                               */
    CUTS_EOVERFLOW = -4,    /* count >= 2^64 (cuts_count); full value in cuts_stats     */
    CUTS_ETRUNC = -5,       /* enumeration found more rows than cap_rows                */
    CUTS_ESTATE = -6,       /* call out of order                                        */
    CUTS_EUNSUPPORTED = -7, /* k > 8                                                    */
    CUTS_ECOMM = -8         /* NCCL / donation transport failure (multi-GPU layer)      */
} cuts_status;

typedef enum {
    CUTS_BFS = 0,    /* level-synchronous: every level stored whole (Alg. 1);
                        CUTS_ENOMEM when a level does not fit the arena                    */
    CUTS_HYBRID = 1  /* BFS inside chunks, DFS over chunks      */
} cuts_mode;

typedef struct {
    int       device;       /* CUDA device ordinal                                          */
    uintptr_t stream;       /* cudaStream_t (e.g. torch.cuda.current_stream().cuda_stream) */
    void*     arena;        /* caller-owned device scratch: degrees, trie levels, counters  */
    uint64_t  arena_bytes;  /* hard budget (the paper uses 1/2 of free memory per array,
                               P:688-691); >= 256-byte aligned base required               */
    uint64_t  seed;         /* level-1 shuffle; never changes any result        */
} cuts_opts;

typedef struct {
    uint32_t k;                        /* query size                                        */
    uint32_t order[CUTS_MAX_K];        /* matching order S actually used                    */
    uint64_t level_size[CUTS_MAX_K + 1];  /* |L_j| summed over chunks, j = 0..k; L_k = count
                                          (low 64 bits); exact and chunk-invariant          */
    uint64_t count_lo, count_hi;       /* 128-bit embedding count                           */
    uint64_t level1_canonical;         /* size of the canonical level-1 list (deg filter)   */
    uint64_t chunks;                   /* extend launches (hybrid chunks x windows)         */
    uint64_t windows;                  /* plan windows                                      */
    uint64_t launches;                 /* kernels launched by the last count/enumerate      */
    uint64_t peak_arena_bytes;         /* high-water mark of the arena stack                */
    uint64_t items;                    /* candidate items examined (sum of min list sizes)  */
    double   ms_total;                 /* host wall time of the call                        */
    double   ms_extend;                /* device time of extend/count kernels (if timing)   */
    double   ms_plan;                  /* device time of plan + scan kernels (if timing)    */
    uint64_t extend_launches;          /* launches timed in ms_extend                       */
    uint64_t alg_bytes_extend;         /* algorithmic bytes of the extend kernels, SURVEY §8.d
                                          model kept FIXED: 4 d per backward list of every
                                          entry + 4 per intersection survivor + children
                                          written (only with CUTS_DEBUG_BYTES)              */
    uint64_t alg_bytes_plan;           /* algorithmic bytes of the plan kernels (ditto)     */
    uint64_t hubs;                     /* vertices with an adjacency bitmap (see below)     */
    uint64_t hub_threshold;            /* degree threshold used for the bitmaps             */
    uint64_t donations;                /* work donations made (cuts_set_donation)           */
    uint64_t donated_entries;          /* prefixes given away by those donations            */
    uint64_t alg_bytes_extend_needed;  /* bytes the extend path's own algorithm needs (source
                                          actually streamed: shortest list, ancestor range or
                                          set-difference searches; + output) — beside the
                                          frozen §8.d model in alg_bytes_extend              */
    uint64_t free_identity;            /* disconnected Q: 1 if the component roots streamed the
                                          identity list [0, n) with an in-kernel degree
                                          filter (the filtered lists did not fit the arena)  */
    uint64_t fused_levels;             /* bit j: level j was (at least partly) never stored —
                                          the local-rows tail counts it from the level j-1
                                          sibling rows (level_size[j] stays exact)           */
    double   ms_tail;                  /* CUTS_DEBUG_TIMING: CUDA-event ms of the deep-local-
                                          rows tail kernel (k_dlr_tail) alone                */
    uint64_t tail_launches;            /* launches timed in ms_tail                         */
    uint64_t tail_word_ops;            /* CUTS_DEBUG_BYTES: 64-bit AND+POPC word operations
                                          of the tail's bit algebra (its ALU roofline unit)  */
} cuts_stats;

/* debug / instrumentation flags for cuts_set_debug */
#define CUTS_DEBUG_TIMING 1u   /* CUDA events around each kernel -> ms_extend / ms_plan     */
#define CUTS_DEBUG_BYTES  2u   /* per-warp algorithmic byte counters (perturbs timing)      */
#define CUTS_DEBUG_NO_REUSE 4u /* HYBRID: disable the ancestor-set source (ablation); BFS
                                  mode never uses it                                        */
#define CUTS_DEBUG_NO_PACK  8u /* at the next cuts_load_graph: no packed (id | degree) copy
                                  of col in the arena (ablation)                            */
#define CUTS_DEBUG_FIRST_SOURCE 16u /* ablation (NEXT-2): stream the FIRST backward list as
                                  Alg. 2 l.22-23 does (a1) instead of the shortest one      */
#define CUTS_DEBUG_NO_FAST_COUNT 32u /* ablation: stream the list at a single-list,
                                  degree-free last level of cuts_count instead of counting
                                  |list| - |path found in list| by binary search            */
#define CUTS_DEBUG_PRELOAD_COUNT 64u /* test hook: cuts_count starts its 128-bit counter at
                                  2^64 - 2^20 instead of 0 (exercises the carry into the
                                  high word and CUTS_EOVERFLOW; the result is offset)      */
#define CUTS_DEBUG_BINNED 128u /* ablation (NEXT-2): the last level groups its entries into
                                  bins by work and runs each bin with its own virtual-warp
                                  width instead of one bin sized by the average
                                  (the paper's choice)                          */
#define CUTS_DEBUG_SV 256u     /* ablation (NEXT-2): scatter-vector intersection (Alg. 2
                                  l.7-17) with a u8 sv[n] per warp in the arena,
                                  CSR lists only (no hub bitmaps, no ancestor source, no
                                  set-difference count); undirected; count/write modes      */
#define CUTS_DEBUG_NO_PAIRS 512u /* ablation: at a count-only last level whose only list left
                                  besides the ancestor range is the entry's own adjacency
                                  (cliques), test every sibling pair from both ends instead
                                  of once (the default shares each unordered pair)         */
#define CUTS_DEBUG_NO_LR 1024u /* ablation: no local rows — the last two levels of a
                                  clique-like tail go through the trie pipeline (ordered
                                  write of level k-1, pair count) instead of 64-bit sibling
                                  adjacency rows of the level-(k-2) groups                  */
#define CUTS_DEBUG_NO_DLR 4096u /* ablation: no deep local rows — the last three levels of a
                                  clique-like count go through the ordered level-(k-3)
                                  extension and the (k-2)-level local rows instead of the
                                  level-(k-3) sibling rows carrying all three              */
#define CUTS_DEBUG_TAIL_ALT 8192u /* ablation: the deep-local-rows tail gives one lane per
                                  triangle (warp scan + shuffle search) instead of one lane
                                  per level-(k-2) entry                                     */
#define CUTS_DEBUG_TAIL_SPLIT 16384u /* experiment: the tail queues entries split into
                                  work items of 8 triangles                                 */
#define CUTS_DEBUG_NO_CTA_TAIL 32768u /* ablation: the deep-rows tail of wide-row groups
                                  (W >= 2) stays in the warp-queue kernel instead of a CTA per
                                  group with its rows staged in shared memory by TMA        */
#define CUTS_DEBUG_GROUPS 2048u /* instrumentation: histogram of sibling-group sizes (children
                                  per entry) of every ordered level, read with
                                  cuts_debug_group_hist                                     */

/* Create a context bound to opts->device / opts->stream / opts->arena.
 * CUTS_EINVAL if out/opts is NULL, arena is NULL or misaligned, or arena_bytes < 64 KiB. */
cuts_status cuts_create(cuts_ctx** out, const cuts_opts* opts);

/* Release host resources of ctx (the caller's device buffers are untouched). NULL-safe. */
void cuts_destroy(cuts_ctx* ctx);

/* Message for the last failing call on ctx (never NULL; "" after success). */
const char* cuts_last_error(const cuts_ctx* ctx);

/* ABI version (CUTS_ABI_VERSION). */
int cuts_version(void);

/* Data graph D as symmetric CSR (undirected edges stored both ways,
 * P:207-209): d_row_ptr u64[n+1], d_col u32[nnz], DEVICE pointers borrowed until
 * cuts_destroy or the next load.  Rows strictly ascending, no self loops, ids < n.
 * Derives deg u32[n] into the arena.  validate != 0 runs a device check and
 * returns CUTS_EINVAL on asymmetry, unsorted rows, duplicates, loops or bad ids. */
cuts_status cuts_load_graph(cuts_ctx* ctx, uint32_t n, uint64_t nnz,
                            const uint64_t* d_row_ptr, const uint32_t* d_col, int validate);

/* Directed data graph ("we consider directed graphs"; NEXT-1) as ONE
 * DEVICE CSR of 2n rows: rows 0..n-1 are the out-lists (children, the paper's
 * D.cs), rows n..2n-1 the in-lists (parents, D.ps, used by the p-intersection
 * of Alg. 2 l.33-42).  d_row_ptr u64[2n+1], d_col u32[nnz] with
 * nnz = 2 x arcs; every row strictly ascending, ids < n, no loops; the in-rows
 * must be the transpose of the out-rows (checked when validate != 0, else
 * CUTS_EINVAL).  2n < 2^32-1.  Borrowed like cuts_load_graph's arrays.  Hub
 * bitmaps and the packed candidate stream are not used for directed graphs.
 * Pair with cuts_set_query_directed (an undirected query on a directed graph,
 * or the reverse, fails at count time with CUTS_EINVAL). */
cuts_status cuts_load_digraph(cuts_ctx* ctx, uint32_t n, uint64_t nnz,
                              const uint64_t* d_row_ptr, const uint32_t* d_col, int validate);

/* Membership rows for hub vertices (SV-style intersection, Alg. 2 l.7-17,
 * P:1055-1072): at the next cuts_load_graph, every vertex with deg >= t gets a
 * bitmap of its neighbours over [0, n) in the arena, and a membership test
 * against its list becomes one load.  t = 0: automatic (the smallest power of
 * two >= 256 whose bitmaps fit min(arena/16, 8 GiB)); t = UINT32_MAX: off.
 * Never changes a result.  Default 0. */
cuts_status cuts_set_hub_threshold(cuts_ctx* ctx, uint32_t t);

/* Query Q as HOST CSR over 0..k-1 (1 <= k <= 8): row_ptr u32[k+1], col u32[...],
 * symmetric, no loops/duplicates.  Q may be disconnected: the result
 * is the cross product of the components' embeddings restricted to injective
 * combinations (reading P16), built inside the same trie — a component's first
 * matched vertex (bw = 0) takes its candidates from {v : deg(v) >= its degree}
 * and the injectivity filter removes the overlapping combinations.
 * order == NULL -> the paper's rule: root = max degree (ties: min id),
 * then the max-degree vertex adjacent to the matched set (ties: min
 * id, reading P6); when no unmatched vertex touches the matched set, the next
 * component starts at its max-degree vertex (ties: min id).  Else order is a
 * permutation of 0..k-1 in which every order[i], i >= 1, has a neighbour in
 * order[0..i-1] or is the first of its component (else CUTS_EINVAL).
 * Resets the root range and partition to "all". */
cuts_status cuts_set_query(cuts_ctx* ctx, uint32_t k, const uint32_t* row_ptr,
                           const uint32_t* col, const uint32_t* order);

/* Directed query Q as HOST out-CSR over 0..k-1 (row_ptr u32[k+1], col u32:
 * arcs a -> col[p]), no loops/duplicate arcs.  Embeddings are the injective f
 * with (u,w) in arcs(Q) => (f(u),f(w)) in arcs(D) (reading P1, directed).
 * Degree filter: outdeg(c) >= outdeg_Q and indeg(c) >= indeg_Q (Def. 5 with the
 * in/out degree of P:262-264; reading P27).  order == NULL -> root = max
 * out-degree (ties min id), then the max out-degree vertex weakly
 * adjacent to the matched set; weak components in turn.  A position
 * whose backward arcs need more lists than its index (reciprocal query arcs
 * u <-> w at that position) returns CUTS_EUNSUPPORTED. */
cuts_status cuts_set_query_directed(cuts_ctx* ctx, uint32_t k, const uint32_t* row_ptr,
                                    const uint32_t* col, const uint32_t* order);

/* Restrict the roots to positions [begin, end) of the CANONICAL level-1 list
 * (vertices with deg >= deg_Q(S[0]) in ascending id, before shuffling; Alg. 1
 * l.8-11).  end is clamped to the list size.  Default: all. */
cuts_status cuts_set_root_range(cuts_ctx* ctx, uint64_t begin, uint64_t end);

/* Select a slice of the SHUFFLED level-1 list (after the root range): positions
 * p in [begin, end) with p % nparts == part.  This is the multi-GPU partition
 * point (|V_D|/nGPU roots per GPU) and the unit of the dynamic
 * root-chunk queue.  Default: begin = 0, end = UINT64_MAX, part = 0, nparts = 1. */
cuts_status cuts_set_root_slice(cuts_ctx* ctx, uint64_t begin, uint64_t end,
                                uint32_t part, uint32_t nparts);

/* Size of the level-1 candidate list for the current query (runs the device
 * degree-filter compaction, Alg. 1 l.8-11): *canonical = |{u : deg(u) >=
 * deg_Q(S[0])}|, *in_range = how many of those lie in the root range (the
 * length of the shuffled list that cuts_set_root_slice positions index).
 * Either pointer may be NULL. */
cuts_status cuts_level1_size(cuts_ctx* ctx, uint64_t* canonical, uint64_t* in_range);

/* Exact number of ordered non-induced embeddings of Q in D restricted to the
 * selected roots.  *out = low 64 bits; CUTS_EOVERFLOW if the count is >= 2^64
 * (full 128-bit value in cuts_stats).  mode: CUTS_BFS or CUTS_HYBRID. */
cuts_status cuts_count(cuts_ctx* ctx, cuts_mode mode, uint64_t* out);

/* Enumerate embeddings into d_out (DEVICE, cap_rows * k u32): row[q] = f(q) in
 * QUERY-VERTEX-ID order; row order unspecified (any trie order is valid,
 * P:700-703).  *n_found is exact; if > cap_rows -> CUTS_ETRUNC and which rows
 * were written is unspecified. */
cuts_status cuts_enumerate(cuts_ctx* ctx, cuts_mode mode, uint32_t* d_out,
                           uint64_t cap_rows, uint64_t* n_found);

/* Multi-GPU partition below level 1 (an extension of the paper's first-level partition,
 * P:1277-1279, for power-law roots whose subtrees differ by orders of magnitude): with
 * depth D > 1 every count/enumerate builds levels 1..D whole over the root range (BFS,
 * identical on every part), shuffles level D with the seeded bijection and
 * applies the cuts_set_root_slice (begin, end, part, nparts) — or the cuts_set_dist
 * default — to THAT list, then extends the slice (HYBRID or BFS) from flat prefixes.
 * Summed over the parts of a partition the counts equal the unpartitioned count and the
 * level sizes are exact (levels < D are reported by the part holding shuffled position 0
 * only).  D = 1 (default) slices the level-1 list; D >= k behaves like 1.  CUTS_EINVAL
 * unless 1 <= D < 8.  Persists across queries. */
cuts_status cuts_set_partition_depth(cuts_ctx* ctx, uint32_t depth);

/* Size of the list the slice partitions: |L_D| over the root range for the current
 * query and partition depth (|L_1| in range for D = 1); runs the BFS to level D. */
cuts_status cuts_partition_size(cuts_ctx* ctx, uint64_t* n);

/* Stats of the last count/enumerate. */
cuts_status cuts_get_stats(const cuts_ctx* ctx, cuts_stats* out);

/* Instrumentation flags (CUTS_DEBUG_*); 0 for the timed product path. */
cuts_status cuts_set_debug(cuts_ctx* ctx, uint32_t flags);

/* CUTS_DEBUG_GROUPS result of the last count: out[(j * 16 + b) * 3 + {0, 1, 2}] =
 * number of level-j sibling groups (the children of one level-(j-1) entry, written
 * ordered) with size m in bucket b (b = 0: m = 0; b >= 1: 2^(b-1) <= m < 2^b, b = 15
 * holds m >= 2^14), their sum of m, and their sum of m^2; j = 0..8.  out: HOST
 * array of CUTS_GROUP_HIST_WORDS u64.  Zeros when the flag was off. */
#define CUTS_GROUP_HIST_WORDS 432
cuts_status cuts_debug_group_hist(cuts_ctx* ctx, uint64_t* out);

/* Seed the search with flat prefixes instead of level 1 (the receiving side of
 * the dynamic redistribution of Alg. 3, P:1110-1144 l.16-20, "adjust depth",
 * reading P24): d_prefixes is a DEVICE array of count rows of depth u32, row
 * i = (f(S[0]), ..., f(S[depth-1])) in MATCHING-ORDER positions (the order in
 * cuts_stats.order), each a partial embedding of Q[S[0..depth-1]] that passes
 * the degree filter — e.g. rows shipped by a donor's cuts_ship_fn for the same
 * graph and query.  Borrowed until the next count/enumerate returns.  The next
 * count/enumerate extends exactly these prefixes (root range and slice are
 * ignored).  1 <= depth < k, else CUTS_EINVAL; depth == 0 restores level-1
 * seeding.  Reset by cuts_set_query.  Rows that are not valid partial
 * embeddings give an unspecified count. */
cuts_status cuts_set_prefixes(cuts_ctx* ctx, uint32_t depth, uint64_t count,
                              const uint32_t* d_prefixes);

/* Donation hooks (the sending side of Alg. 3).  In CUTS_HYBRID
 * runs the library calls poll(user, depth, remaining) at every chunk boundary,
 * where depth is the shallowest level of the DFS stack with at least two
 * entries not yet started and remaining their number; poll returns how many of them to give
 * away (0: none; clamped to remaining).  The library then exports the LAST
 * `give` of those entries as flat prefixes (rows of depth u32, matching-order
 * positions, format of cuts_set_prefixes) into arena scratch, synchronises its
 * stream and calls ship(user, depth, d_prefixes, give); the buffer is valid
 * only during the call (copy it out); if the arena has no room for the rows,
 * ship is called with d_prefixes = NULL and count = 0 instead.  A non-zero return from ship aborts the
 * count with CUTS_ECOMM.  The donated entries are never extended here, so the
 * local count excludes them.  Both NULL (default): no donation.  Callbacks run
 * on the calling thread. */
typedef uint64_t (*cuts_poll_fn)(void* user, uint32_t depth, uint64_t remaining);
typedef int (*cuts_ship_fn)(void* user, uint32_t depth, const uint32_t* d_prefixes, uint64_t count);
cuts_status cuts_set_donation(cuts_ctx* ctx, cuts_poll_fn poll, cuts_ship_fn ship, void* user);

/* Decode a trie (Fig. 3C) held in DEVICE memory: level l (0-based,
 * l < nlevels <= 8) has sizes[l] entries, candidate ids d_ca[l][x] and parent
 * indices d_pa[l][x] into level l-1 (d_pa[0] ignored).  Writes, for every entry
 * x of the last level, the root-to-leaf path as nlevels u32 at d_out[x*nlevels].
 * sizes / d_ca / d_pa are HOST arrays of length nlevels.  Runs on ctx's stream;
 * CUTS_EINVAL on a parent index out of range. */
cuts_status cuts_trie_decode(cuts_ctx* ctx, uint32_t nlevels, const uint64_t* sizes,
                             const uint32_t* const* d_ca, const uint32_t* const* d_pa,
                             uint32_t* d_out);

/* ------------------------------------------------------------ multi-GPU
 * Row e of the hot path (Alg. 3): one
 * process per GPU, D replicated on every rank (Alg. 3 gives every rank Q and
 * D), level-1 roots partitioned, counts summed with one NCCL
 * all-reduce (the path's only collective).  NCCL is resolved at run time
 * (dlopen of libnccl.so.2, normally the copy torch already loaded); the
 * single-GPU path never needs it. */
#define CUTS_DIST_UID_BYTES 128

/* Write a fresh ncclUniqueId (CUTS_DIST_UID_BYTES bytes) to the HOST buffer
 * out_128B — call on one rank and broadcast it (e.g. torch.distributed).
 * CUTS_ECOMM if NCCL cannot be loaded. */
cuts_status cuts_dist_unique_id(void* out_128B);

/* Join ctx to a world of `world` ranks as `rank` (collective: every rank calls
 * it with the same id).  nccl_uid_128B: HOST copy of the id from
 * cuts_dist_unique_id (may be NULL only when world == 1: no communicator).
 * peers: reserved for peer-mapped donation inboxes, must be NULL (donated
 * prefixes travel through the caller's transport, see cuts_set_donation).
 * Afterwards the default root partition of every query (set by
 * cuts_set_query, overridable with cuts_set_root_slice) is this rank's
 * cyclic slice p % world == rank of the shuffled level-1 list.
 * CUTS_EINVAL on bad rank/world, CUTS_ECOMM if NCCL fails. */
cuts_status cuts_set_dist(cuts_ctx* ctx, int rank, int world, const void* nccl_uid_128B, const void* peers);

/* Collective exact sum over the ranks of a 128-bit count (lo, hi) -> (*out_lo,
 * *out_hi), e.g. the per-rank results of cuts_count: four 32-bit limbs in u64
 * words, one ncclAllReduce(ncclUint64, ncclSum) on ctx's stream.
 * Without a communicator (world == 1) it copies.  Host-synchronous. */
cuts_status cuts_allreduce_count(cuts_ctx* ctx, uint64_t lo, uint64_t hi, uint64_t* out_lo, uint64_t* out_hi);

#ifdef __cplusplus
}
#endif
#endif /* CUTS_H */
