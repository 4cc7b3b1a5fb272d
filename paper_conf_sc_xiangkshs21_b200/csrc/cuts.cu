// cuts.cu — host driver + C ABI of libcuts.so (see include/cuts.h).
// "P:n" cites /root/reference/PAPER.md line n.  Design: DESIGN.md §4-§5.
//
// Memory: everything lives in the caller's arena (P:688-691 uses two halves of
// cudaMemGetInfo's free space; here the caller decides the budget):
//   [ctrl block | deg u32[n] | bottom stack ->  ...free...  <- top stack]
// The bottom stack holds trie levels (persistent while a chunk is being
// expanded), the top stack holds per-depth window scratch (path, source list,
// item offsets, scan temp).  HYBRID mode is a DFS over item-range chunks with
// BFS inside each chunk; BFS mode stores each level whole.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>   // types and enum values only: the functions are resolved at run time (dlsym)
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>
#include <thrust/iterator/counting_iterator.h>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "cuts.h"
#include "kernels.cuh"

using namespace cuts;

namespace {

constexpr uint64_t kAlign = 256;
constexpr uint64_t kCtrlBytes = 4096;
constexpr uint64_t kMaxWindow = 1ull << 24;      // entries per plan window
constexpr uint64_t kMaxLevel = 0xFFFFFFFFull;    // u32 parent indices
constexpr uint64_t kPreloadCount = 0xFFFFFFFFFFF00000ull;   // CUTS_DEBUG_PRELOAD_COUNT: 2^64 - 2^20

inline uint64_t align_up(uint64_t x) { return (x + kAlign - 1) & ~(kAlign - 1); }

}  // namespace

struct cuts_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    char* arena = nullptr;
    uint64_t arena_bytes = 0;
    uint64_t seed = 0;
    std::string err;
    int num_sms = 148;
    unsigned long long* ctrl = nullptr;   // device control words
    unsigned long long* h_ctrl = nullptr; // pinned host mirror
    // graph
    bool has_graph = false;
    bool directed = false;                 // cuts_load_digraph: 2n rows (out-lists, then in-lists)
    uint32_t n = 0;
    uint64_t nnz = 0;
    const uint64_t* row_ptr = nullptr;
    const uint32_t* col = nullptr;
    uint32_t* deg = nullptr;
    uint32_t* hub = nullptr;               // hub[v] -> bitmap row, or kNoHub
    uint32_t* bm = nullptr;                // hub bitmaps
    uint32_t* cb = nullptr;                // hub-to-hub core bitmap (nhubs^2 bits)
    uint32_t cbw = 0;
    uint32_t* colx = nullptr;              // packed (id | min(deg,31) << 27) copy of col, or null
    uint32_t words = 0;
    uint64_t nhubs = 0, hub_t_used = 0;
    uint32_t hub_t = 0;                    // requested threshold (0 auto, UINT32_MAX off)
    uint64_t base_off = 0;                 // first free byte after ctrl + deg + bitmaps
    // canonical level-1 list of the current query (Alg. 1 l.8-11), built once per
    // (graph, query) right after base_off and reused by every count / root chunk
    bool canon_valid = false;
    uint32_t* canon = nullptr;
    uint64_t canon_n = 0;
    uint64_t run_off = 0;                  // first free byte after the canonical list
    // query
    bool has_query = false;
    bool q_directed = false;
    QPlan q{};
    uint64_t root_begin = 0, root_end = ~0ull;
    uint64_t slice_begin = 0, slice_end = ~0ull;
    uint32_t part = 0, nparts = 1;
    uint32_t part_depth = 1;               // level whose shuffled list the slice partitions
    bool size_only = false;                // cuts_partition_size: stop after the partition level
    uint32_t debug = 0;
    // run state
    uint64_t bot = 0, top = 0, peak = 0;
    cuts_stats st{};
    int extend_occ_blocks = 0;
    std::vector<cudaEvent_t> ev_pool;
    size_t ev_used = 0;
    std::vector<std::pair<int, int>> ev_ext, ev_plan, ev_tail;
    // flat-prefix seeding (cuts_set_prefixes): run from level pre_j instead of level 1
    uint32_t pre_j = 0;
    uint64_t pre_count = 0;
    const uint32_t* pre_rows = nullptr;
    // work donation (cuts_set_donation): DFS cursor per depth of the HYBRID stack
    cuts_poll_fn poll = nullptr;
    cuts_ship_fn ship = nullptr;
    void* user = nullptr;
    // ancestor-set reuse: anc[J] = ancestor level whose children range
    // sources level J's candidates (0: none); bit a of need_ord: level a -> a+1 is
    // written ordered (children contiguous per parent, exact offsets kept)
    uint32_t anc[kMaxK + 1] = {};
    uint32_t need_ord = 0;
    struct OrdState { const uint64_t* cpos; uint64_t w0; uint64_t ea; const uint2* lv; bool valid; uint64_t eb; };
    OrdState ord[kMaxK + 1] = {};
    // CUTS_DEBUG_SV: per-warp u8 scatter vectors of n entries (zeroed; kernels leave them clean)
    uint8_t* sv = nullptr;
    uint64_t sv_warps = 0;
    // multi-GPU (cuts_set_dist): rank / world and the NCCL communicator of the count reduction
    int rank = 0, world = 1;
    ncclComm_t comm = nullptr;
    uint64_t dfs_next[kMaxK + 1] = {};   // first entry of level d not yet planned
    uint64_t dfs_end[kMaxK + 1] = {};    // end of level d's entries still owned here
    bool dfs_on[kMaxK + 1] = {};
};

namespace {

// NCCL through dlopen: the process normally has it loaded already (torch's
// libnccl.so.2), so RTLD_NOLOAD reuses that copy; libcuts.so has no link-time
// NCCL dependency and the single-GPU path never touches it.
struct NcclApi {
    decltype(&ncclGetUniqueId) get_unique_id = nullptr;
    decltype(&ncclCommInitRank) init_rank = nullptr;
    decltype(&ncclAllReduce) all_reduce = nullptr;
    decltype(&ncclCommDestroy) destroy = nullptr;
    decltype(&ncclGetErrorString) error_string = nullptr;
    bool tried = false, ok = false;
};

NcclApi& nccl() {
    static NcclApi api;
    if (api.tried) return api;
    api.tried = true;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return api;
    api.get_unique_id = (decltype(api.get_unique_id))dlsym(h, "ncclGetUniqueId");
    api.init_rank = (decltype(api.init_rank))dlsym(h, "ncclCommInitRank");
    api.all_reduce = (decltype(api.all_reduce))dlsym(h, "ncclAllReduce");
    api.destroy = (decltype(api.destroy))dlsym(h, "ncclCommDestroy");
    api.error_string = (decltype(api.error_string))dlsym(h, "ncclGetErrorString");
    api.ok = api.get_unique_id && api.init_rank && api.all_reduce && api.destroy && api.error_string;
    return api;
}

cuts_status fail(cuts_ctx* c, cuts_status s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) c->err = buf;
    return s;
}

#define CK(call)                                                                               \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess)                                                                 \
            return fail(ctx, CUTS_ECUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), \
                        __FILE__, __LINE__);                                                   \
    } while (0)

#define TRY(expr)                         \
    do {                                  \
        cuts_status s_ = (expr);          \
        if (s_ != CUTS_OK) return s_;     \
    } while (0)

// ---- arena stacks --------------------------------------------------------
cuts_status alloc_bot(cuts_ctx* ctx, uint64_t bytes, uint64_t* off) {
    uint64_t b = align_up(ctx->bot);
    if (b + bytes > ctx->top) return fail(ctx, CUTS_ENOMEM, "arena exhausted (bottom stack needs %llu B)", (unsigned long long)bytes);
    *off = b;
    ctx->bot = b + bytes;
    ctx->peak = std::max(ctx->peak, ctx->bot + (ctx->arena_bytes - ctx->top));
    return CUTS_OK;
}
cuts_status alloc_top(cuts_ctx* ctx, uint64_t bytes, uint64_t* off) {
    uint64_t need = align_up(bytes);
    if (ctx->top < need || ctx->top - need < align_up(ctx->bot))
        return fail(ctx, CUTS_ENOMEM, "arena exhausted (top stack needs %llu B)", (unsigned long long)bytes);
    ctx->top -= need;
    *off = ctx->top;
    ctx->peak = std::max(ctx->peak, ctx->bot + (ctx->arena_bytes - ctx->top));
    return CUTS_OK;
}
inline uint64_t free_bytes(const cuts_ctx* ctx) {
    uint64_t b = align_up(ctx->bot);
    return ctx->top > b ? ctx->top - b : 0;
}

// ---- events --------------------------------------------------------------
int next_event(cuts_ctx* ctx) {
    if (ctx->ev_used == ctx->ev_pool.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return -1;
        ctx->ev_pool.push_back(e);
    }
    return (int)ctx->ev_used++;
}

// ---- query planning --------------------------------
bool q_adj(const uint32_t* row, const uint32_t* col, uint32_t a, uint32_t b) {
    for (uint32_t p = row[a]; p < row[a + 1]; ++p)
        if (col[p] == b) return true;
    return false;
}

cuts_status plan_query(cuts_ctx* ctx, uint32_t k, const uint32_t* row, const uint32_t* col,
                       const uint32_t* order, QPlan* out) {
    if (k < 1 || k > CUTS_MAX_K) return fail(ctx, k > CUTS_MAX_K ? CUTS_EUNSUPPORTED : CUTS_EINVAL, "k=%u out of range 1..8", k);
    if (!row || (row[k] > 0 && !col)) return fail(ctx, CUTS_EINVAL, "null query arrays");
    if (row[0] != 0) return fail(ctx, CUTS_EINVAL, "query row_ptr[0] != 0");
    for (uint32_t a = 0; a < k; ++a) {
        if (row[a + 1] < row[a]) return fail(ctx, CUTS_EINVAL, "query row_ptr not monotone");
        for (uint32_t p = row[a]; p < row[a + 1]; ++p) {
            uint32_t b = col[p];
            if (b >= k || b == a) return fail(ctx, CUTS_EINVAL, "query edge (%u,%u) invalid", a, b);
            for (uint32_t p2 = row[a]; p2 < p; ++p2)
                if (col[p2] == b) return fail(ctx, CUTS_EINVAL, "duplicate query edge (%u,%u)", a, b);
            if (!q_adj(row, col, b, a)) return fail(ctx, CUTS_EINVAL, "query not symmetric at (%u,%u)", a, b);
        }
    }
    // connected components: comp[a] = smallest vertex of a's component
    uint32_t comp[CUTS_MAX_K];
    for (uint32_t a = 0; a < k; ++a) comp[a] = a;
    for (bool changed = true; changed;) {
        changed = false;
        for (uint32_t a = 0; a < k; ++a)
            for (uint32_t p = row[a]; p < row[a + 1]; ++p)
                if (comp[col[p]] < comp[a]) { comp[a] = comp[col[p]]; changed = true; }
    }
    uint32_t S[CUTS_MAX_K];
    auto qdeg = [&](uint32_t a) { return row[a + 1] - row[a]; };
    if (order) {
        uint32_t used = 0;
        for (uint32_t i = 0; i < k; ++i) {
            if (order[i] >= k || (used >> order[i] & 1u)) return fail(ctx, CUTS_EINVAL, "order is not a permutation");
            used |= 1u << order[i];
            S[i] = order[i];
        }
    } else {
        // root: max degree, ties -> min id; then max degree adjacent
        // to the matched set, ties -> min id (reading P6).  When no
        // unmatched vertex touches the matched set, the next component starts
        // at its max-degree vertex (components in turn, reading P16)
        uint32_t used = 0;
        for (uint32_t i = 0; i < k; ++i) {
            int pick = -1;
            for (int pass = 0; pass < 2 && pick < 0; ++pass) {
                for (uint32_t a = 0; a < k; ++a) {
                    if (used >> a & 1u) continue;
                    bool touches = (i == 0) || pass == 1;
                    for (uint32_t j = 0; j < i && !touches; ++j) touches = q_adj(row, col, a, S[j]);
                    if (!touches) continue;
                    if (pick < 0 || qdeg(a) > qdeg((uint32_t)pick)) pick = (int)a;
                }
            }
            S[i] = (uint32_t)pick;
            used |= 1u << pick;
        }
    }
    QPlan qp{};
    qp.k = k;
    for (uint32_t i = 0; i < k; ++i) {
        qp.S[i] = S[i];
        qp.qdeg[i] = qdeg(S[i]);
        qp.bw[i] = 0;
        for (uint32_t j = 0; j < i; ++j)
            if (q_adj(row, col, S[j], S[i])) qp.bw[i] |= 1u << j;
        bool starts = true;   // no earlier position in S[i]'s component
        for (uint32_t j = 0; j < i; ++j) starts = starts && comp[S[j]] != comp[S[i]];
        if (i > 0 && qp.bw[i] == 0 && !starts)
            return fail(ctx, CUTS_EINVAL, "order position %u (query vertex %u) has no backward neighbour", i, S[i]);
    }
    *out = qp;
    return CUTS_OK;
}

// ---- directed query planning (NEXT-1) ---------------------
// Q as out-CSR over 0..k-1.  Order: root = max out-degree ("out degree in the
// case of directed graphs"; ties min id), then the max out-degree vertex
// weakly adjacent to the matched set, a new weak component when none is.
// bw[i] bit p: arc S[p] -> S[i] (children list, c-intersection); bwi[i] bit p:
// arc S[i] -> S[p] (parents list, p-intersection, Alg. 2 l.33-42).
cuts_status plan_query_directed(cuts_ctx* ctx, uint32_t k, const uint32_t* row, const uint32_t* col,
                                const uint32_t* order, QPlan* out) {
    if (k < 1 || k > CUTS_MAX_K) return fail(ctx, k > CUTS_MAX_K ? CUTS_EUNSUPPORTED : CUTS_EINVAL, "k=%u out of range 1..8", k);
    if (!row || (row[k] > 0 && !col)) return fail(ctx, CUTS_EINVAL, "null query arrays");
    if (row[0] != 0) return fail(ctx, CUTS_EINVAL, "query row_ptr[0] != 0");
    for (uint32_t a = 0; a < k; ++a) {
        if (row[a + 1] < row[a]) return fail(ctx, CUTS_EINVAL, "query row_ptr not monotone");
        for (uint32_t p = row[a]; p < row[a + 1]; ++p) {
            if (col[p] >= k || col[p] == a) return fail(ctx, CUTS_EINVAL, "query arc (%u,%u) invalid", a, col[p]);
            for (uint32_t p2 = row[a]; p2 < p; ++p2)
                if (col[p2] == col[p]) return fail(ctx, CUTS_EINVAL, "duplicate query arc (%u,%u)", a, col[p]);
        }
    }
    auto arc = [&](uint32_t a, uint32_t b) { return q_adj(row, col, a, b); };
    auto weak = [&](uint32_t a, uint32_t b) { return arc(a, b) || arc(b, a); };
    auto outd = [&](uint32_t a) { return row[a + 1] - row[a]; };
    uint32_t comp[CUTS_MAX_K];
    for (uint32_t a = 0; a < k; ++a) comp[a] = a;
    for (bool changed = true; changed;) {
        changed = false;
        for (uint32_t a = 0; a < k; ++a)
            for (uint32_t b = 0; b < k; ++b)
                if (weak(a, b) && comp[b] < comp[a]) { comp[a] = comp[b]; changed = true; }
    }
    uint32_t S[CUTS_MAX_K];
    uint32_t used = 0;
    if (order) {
        for (uint32_t i = 0; i < k; ++i) {
            if (order[i] >= k || (used >> order[i] & 1u)) return fail(ctx, CUTS_EINVAL, "order is not a permutation");
            used |= 1u << order[i];
            S[i] = order[i];
        }
    } else {
        for (uint32_t i = 0; i < k; ++i) {
            int pick = -1;
            for (int pass = 0; pass < 2 && pick < 0; ++pass)
                for (uint32_t a = 0; a < k; ++a) {
                    if (used >> a & 1u) continue;
                    bool touches = (i == 0) || pass == 1;
                    for (uint32_t j = 0; j < i && !touches; ++j) touches = weak(a, S[j]);
                    if (!touches) continue;
                    if (pick < 0 || outd(a) > outd((uint32_t)pick)) pick = (int)a;
                }
            S[i] = (uint32_t)pick;
            used |= 1u << pick;
        }
    }
    QPlan qp{};
    qp.k = k;
    for (uint32_t i = 0; i < k; ++i) {
        qp.S[i] = S[i];
        qp.qdeg[i] = outd(S[i]);
        qp.qdin[i] = 0;
        for (uint32_t a = 0; a < k; ++a) qp.qdin[i] += arc(a, S[i]) ? 1u : 0u;
        for (uint32_t j = 0; j < i; ++j) {
            if (arc(S[j], S[i])) qp.bw[i] |= 1u << j;
            if (arc(S[i], S[j])) qp.bwi[i] |= 1u << j;
        }
        bool starts = true;
        for (uint32_t j = 0; j < i; ++j) starts = starts && comp[S[j]] != comp[S[i]];
        const uint32_t nreq = __builtin_popcount(qp.bw[i]) + __builtin_popcount(qp.bwi[i]);
        if (i > 0 && nreq == 0 && !starts)
            return fail(ctx, CUTS_EINVAL, "order position %u (query vertex %u) has no backward neighbour", i, S[i]);
        if (i > 0 && nreq > i)
            return fail(ctx, CUTS_EUNSUPPORTED, "position %u needs %u lists (> %u): reciprocal query arcs at this position "
                        "are not supported", i, nreq, i);
    }
    *out = qp;
    return CUTS_OK;
}

// ---- kernel dispatch -------------------------------------------------------
struct Window {
    uint64_t w0;
    uint32_t W;
    uint32_t* path;
    uint64_t* src;
    uint64_t* lst_off;   // (J-1) x W list descriptors from k_plan
    uint32_t* lst_len;
    uint64_t* cpos;      // ordered levels: exclusive scan of the children per entry (W+1)
    Reuse ru{};          // ancestor-set source for this level (ru.a == 0: off)
    uint64_t* ord_cnt = nullptr;         // pass A output (children per entry)
    const uint64_t* ord_pos = nullptr;   // pass B: exact child offsets
    uint32_t ord_ea = 0;                 // pass B: first entry of the chunk
    uint64_t* ub;
    uint64_t* offs;
    void* cub_tmp;
    size_t cub_bytes;
    uint64_t total;
    const uint32_t* elist = nullptr;     // binned launch: explicit entry list (one bin)
    uint32_t elist_n = 0;
    int force_g = 0;                     // binned launch: that bin's virtual-warp width
};

template <int J>
void launch_plan_t(cuts_ctx* ctx, const Graph& g, const Trie& t, const Window& w, int grid) {
    if (ctx->directed)
        k_plan<J, true><<<grid, 256, 0, ctx->stream>>>(g, t, ctx->q, w.w0, w.W, w.path, w.src, w.ub, w.lst_off, w.lst_len, ctx->ctrl,
                                             (ctx->debug & CUTS_DEBUG_BYTES) ? 1 : 0, w.ru);
    else
        k_plan<J, false><<<grid, 256, 0, ctx->stream>>>(g, t, ctx->q, w.w0, w.W, w.path, w.src, w.ub, w.lst_off, w.lst_len, ctx->ctrl,
                                             (ctx->debug & CUTS_DEBUG_BYTES) ? 1 : 0, w.ru);
}

void launch_plan(cuts_ctx* ctx, int J, const Graph& g, const Trie& t, const Window& w) {
    int grid = (int)std::min<uint64_t>((w.W + 1 + 255) / 256, (uint64_t)ctx->num_sms * 8);
    switch (J) {
        case 1: launch_plan_t<1>(ctx, g, t, w, grid); break;
        case 2: launch_plan_t<2>(ctx, g, t, w, grid); break;
        case 3: launch_plan_t<3>(ctx, g, t, w, grid); break;
        case 4: launch_plan_t<4>(ctx, g, t, w, grid); break;
        case 5: launch_plan_t<5>(ctx, g, t, w, grid); break;
        case 6: launch_plan_t<6>(ctx, g, t, w, grid); break;
        case 7: launch_plan_t<7>(ctx, g, t, w, grid); break;
    }
}

template <int J, int NL, int M, int G>
void launch_extend_g(cuts_ctx* ctx, const Graph& g, const Window& w, uint64_t t0, uint64_t t1,
                     uint2* out_level, uint32_t* out_rows, uint64_t cap) {
    static int occ = 0;
    if (!occ) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_extend<J, NL, M, G>, 256, 0);
        if (occ < 1) occ = 1;
    }
    // persistent-style grid: every resident CTA slot, entries fetched dynamically
    uint64_t need = ((t1 - t0) + 255) / 256 + 1;
    uint64_t grid = std::min<uint64_t>((uint64_t)ctx->num_sms * occ, std::max<uint64_t>(need, 1));
    // entries per virtual-warp fetch: ~2K candidate items per atomic on the work counter
    const double avg = (double)w.total / (double)std::max<uint32_t>(w.W, 1);
    const uint32_t batch = (uint32_t)std::min(256.0, std::max(2.0, 2048.0 / std::max(avg, 1.0) / (32 / G)));
    k_extend<J, NL, M, G><<<(unsigned)grid, 256, 0, ctx->stream>>>(g, ctx->q, w.w0, w.W, w.path, w.src, w.offs,
                                                                   w.lst_off, w.lst_len, t0, t1,
                                                                   out_level, out_rows, cap, ctx->ctrl,
                                                                   (ctx->debug & CUTS_DEBUG_BYTES) && !w.ord_cnt ? 1 : 0, batch,
                                                                   w.ru.a ? ctx->q.qdeg[w.ru.a] : 0u,
                                                                   w.ru.lv, w.ord_cnt, w.ord_pos, w.ord_ea,
                                                                   w.elist, w.elist_n, w.ru.sym ? 2u : 1u,
                                                                   w.ru.sym ? (uint32_t)(J - 1) : 0u);
}

template <int J, int NL, int M>
void launch_extend_nl(cuts_ctx* ctx, const Graph& g, const Window& w, uint64_t t0, uint64_t t1,
                      uint2* out_level, uint32_t* out_rows, uint64_t cap) {
    // virtual-warp width from the average candidate-list length, or the bin's
    const double avg = (double)w.total / (double)std::max<uint32_t>(w.W, 1);
    if (w.force_g == 32) launch_extend_g<J, NL, M, 32>(ctx, g, w, t0, t1, out_level, out_rows, cap);
    else if (w.force_g == 16) launch_extend_g<J, NL, M, 16>(ctx, g, w, t0, t1, out_level, out_rows, cap);
    else if (w.force_g == 8) launch_extend_g<J, NL, M, 8>(ctx, g, w, t0, t1, out_level, out_rows, cap);
    // lanes per entry from the window's average source length (the paper's single bin,
    // P:911-916); thresholds measured on C2 (profiles/r04d_c2_g_*.jsonl: 9.97 -> 9.61 s)
    else if (avg >= 192) launch_extend_g<J, NL, M, 32>(ctx, g, w, t0, t1, out_level, out_rows, cap);
    else if (avg >= 48) launch_extend_g<J, NL, M, 16>(ctx, g, w, t0, t1, out_level, out_rows, cap);
    else launch_extend_g<J, NL, M, 8>(ctx, g, w, t0, t1, out_level, out_rows, cap);
}

// NL = |bw[J]| - 1 lists to test besides the source: a compile-time constant per level
template <int J, int M>
void launch_extend_t(cuts_ctx* ctx, const Graph& g, const Window& w, uint64_t t0, uint64_t t1,
                     uint2* out_level, uint32_t* out_rows, uint64_t cap) {
    // component root: 0; symmetric last level: one list (the entry's own)
    const int nl = w.ru.sym ? 1 : std::max(__builtin_popcount(ctx->q.bw[J]) + __builtin_popcount(ctx->q.bwi[J]) - 1, 0);
    switch (nl) {
        case 0: launch_extend_nl<J, 0, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 1: if constexpr (J > 1) launch_extend_nl<J, (J > 1 ? 1 : 0), M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 2: if constexpr (J > 2) launch_extend_nl<J, (J > 2 ? 2 : 0), M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 3: if constexpr (J > 3) launch_extend_nl<J, (J > 3 ? 3 : 0), M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 4: if constexpr (J > 4) launch_extend_nl<J, (J > 4 ? 4 : 0), M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 5: if constexpr (J > 5) launch_extend_nl<J, (J > 5 ? 5 : 0), M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 6: if constexpr (J > 6) launch_extend_nl<J, (J > 6 ? 6 : 0), M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
    }
}

template <int M>
void launch_extend_m(cuts_ctx* ctx, int J, const Graph& g, const Window& w, uint64_t t0, uint64_t t1,
                     uint2* out_level, uint32_t* out_rows, uint64_t cap) {
    switch (J) {
        case 1: launch_extend_t<1, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 2: launch_extend_t<2, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 3: launch_extend_t<3, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 4: launch_extend_t<4, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 5: launch_extend_t<5, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 6: launch_extend_t<6, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
        case 7: launch_extend_t<7, M>(ctx, g, w, t0, t1, out_level, out_rows, cap); break;
    }
}

template <int J, int NL, int M>
void launch_extend_sv_t(cuts_ctx* ctx, const Graph& g, const Window& w, uint64_t t0, uint64_t t1, uint2* out,
                        uint64_t cap) {
    k_extend_sv<J, NL, M><<<(unsigned)(ctx->sv_warps / 8), 256, 0, ctx->stream>>>(
        g, ctx->q, w.w0, w.W, w.path, w.src, w.offs, w.lst_off, w.lst_len, t0, t1, out, cap, ctx->ctrl, ctx->sv,
        (uint64_t)ctx->n);
}

template <int J, int M>
void launch_extend_sv_j(cuts_ctx* ctx, int nl, const Graph& g, const Window& w, uint64_t t0, uint64_t t1, uint2* out,
                        uint64_t cap) {
    switch (nl) {
        case 1: if constexpr (J > 1) launch_extend_sv_t<J, (J > 1 ? 1 : 1), M>(ctx, g, w, t0, t1, out, cap); break;
        case 2: if constexpr (J > 2) launch_extend_sv_t<J, (J > 2 ? 2 : 1), M>(ctx, g, w, t0, t1, out, cap); break;
        case 3: if constexpr (J > 3) launch_extend_sv_t<J, (J > 3 ? 3 : 1), M>(ctx, g, w, t0, t1, out, cap); break;
        case 4: if constexpr (J > 4) launch_extend_sv_t<J, (J > 4 ? 4 : 1), M>(ctx, g, w, t0, t1, out, cap); break;
        case 5: if constexpr (J > 5) launch_extend_sv_t<J, (J > 5 ? 5 : 1), M>(ctx, g, w, t0, t1, out, cap); break;
        case 6: if constexpr (J > 6) launch_extend_sv_t<J, (J > 6 ? 6 : 1), M>(ctx, g, w, t0, t1, out, cap); break;
    }
}

// SV ablation launch; false if this level has no list to intersect (NL = 0)
template <int M>
bool launch_extend_sv(cuts_ctx* ctx, int J, const Graph& g, const Window& w, uint64_t t0, uint64_t t1, uint2* out,
                      uint64_t cap) {
    const int nl = __builtin_popcount(ctx->q.bw[J]) - 1;
    if (nl < 1) return false;
    switch (J) {
        case 2: launch_extend_sv_j<2, M>(ctx, nl, g, w, t0, t1, out, cap); break;
        case 3: launch_extend_sv_j<3, M>(ctx, nl, g, w, t0, t1, out, cap); break;
        case 4: launch_extend_sv_j<4, M>(ctx, nl, g, w, t0, t1, out, cap); break;
        case 5: launch_extend_sv_j<5, M>(ctx, nl, g, w, t0, t1, out, cap); break;
        case 6: launch_extend_sv_j<6, M>(ctx, nl, g, w, t0, t1, out, cap); break;
        case 7: launch_extend_sv_j<7, M>(ctx, nl, g, w, t0, t1, out, cap); break;
        default: return false;
    }
    return true;
}

// ---- the level pipeline ----------------------------------------------------
struct Run {
    cuts_mode mode;
    bool enumerate;
    uint32_t* rows;
    uint64_t cap_rows;
    Graph g;
    Trie t;
    uint64_t wmax;
};

uint64_t window_scratch_bytes(uint64_t W, int J, size_t cub_bytes) {
    const uint64_t nl = (uint64_t)std::max(J - 1, 1);
    return align_up((uint64_t)J * W * 4) + align_up(W * 8) + 3 * align_up((W + 1) * 8) + align_up(nl * W * 8) +
           align_up(nl * W * 4) + align_up(cub_bytes) + 7 * kAlign;
}

cuts_status read_ctrl(cuts_ctx* ctx) {
    CK(cudaMemcpyAsync(ctx->h_ctrl, ctx->ctrl, kCtrlWords * sizeof(unsigned long long), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return CUTS_OK;
}

// plan window [w0, w0+W) of level J: path walk + ub + scan; sets w.total
cuts_status plan_window(cuts_ctx* ctx, Run& r, int J, Window& w) {
    int e0 = -1, e1 = -1;
    if (ctx->debug & CUTS_DEBUG_TIMING) { e0 = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[e0], ctx->stream)); }
    launch_plan(ctx, J, r.g, r.t, w);
    CK(cudaGetLastError());
    CK(cub::DeviceScan::ExclusiveSum(w.cub_tmp, w.cub_bytes, w.ub, w.offs, (int64_t)w.W + 1, ctx->stream));
    if (ctx->debug & CUTS_DEBUG_TIMING) {
        e1 = next_event(ctx);
        CK(cudaEventRecord(ctx->ev_pool[e1], ctx->stream));
        ctx->ev_plan.push_back({e0, e1});
    }
    CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords, w.offs + w.W, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    w.total = ctx->h_ctrl[kCtrlWords];
    ctx->st.windows++;
    ctx->st.launches += 2;
    ctx->st.items += w.total;
    return CUTS_OK;
}

cuts_status extend_range(cuts_ctx* ctx, Run& r, int J, const Window& w, uint64_t t0, uint64_t t1, int mode,
                         uint2* out, uint64_t cap) {
    if (t1 <= t0) return CUTS_OK;
    int e0 = -1;
    CK(cudaMemsetAsync(ctx->ctrl + kWork, 0, sizeof(unsigned long long), ctx->stream));
    if (ctx->debug & CUTS_DEBUG_TIMING) { e0 = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[e0], ctx->stream)); }
    const bool sv = ctx->sv && mode != kEnum && !w.ord_cnt && !w.ord_pos && !w.elist &&
                    (mode == kWrite ? launch_extend_sv<kWrite>(ctx, J, r.g, w, t0, t1, out, cap)
                                    : launch_extend_sv<kCount>(ctx, J, r.g, w, t0, t1, nullptr, 0));
    if (sv) {
    } else if (mode == kWrite) launch_extend_m<kWrite>(ctx, J, r.g, w, t0, t1, out, nullptr, cap);
    else if (mode == kCount) launch_extend_m<kCount>(ctx, J, r.g, w, t0, t1, nullptr, nullptr, 0);
    else launch_extend_m<kEnum>(ctx, J, r.g, w, t0, t1, nullptr, r.rows, r.cap_rows);
    CK(cudaGetLastError());
    if (ctx->debug & CUTS_DEBUG_TIMING) {
        int e1 = next_event(ctx);
        CK(cudaEventRecord(ctx->ev_pool[e1], ctx->stream));
        ctx->ev_ext.push_back({e0, e1});
    }
    ctx->st.chunks++;
    ctx->st.launches++;
    return CUTS_OK;
}

// last level over the whole window: one launch with the window's single-bin
// virtual warp (the paper's choice), or with CUTS_DEBUG_BINNED one
// launch per non-empty bin of entries grouped by work
cuts_status extend_last(cuts_ctx* ctx, Run& r, int J, const Window& w, int mode) {
    if (!(ctx->debug & CUTS_DEBUG_BINNED) || w.total == 0)
        return extend_range(ctx, r, J, w, 0, w.total, mode, nullptr, 0);
    const uint64_t top_save = ctx->top;
    uint64_t off;
    TRY(alloc_top(ctx, 3ull * w.W * 4, &off));
    uint32_t* bins = (uint32_t*)(ctx->arena + off);
    CK(cudaMemsetAsync(ctx->ctrl + kBins, 0, 3 * sizeof(unsigned long long), ctx->stream));
    const unsigned grid = (unsigned)std::min<uint64_t>((w.W + 255) / 256, (uint64_t)ctx->num_sms * 8);
    k_bin<<<grid, 256, 0, ctx->stream>>>(w.ub, w.W, bins, ctx->ctrl + kBins);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(ctx->h_ctrl + kBins, ctx->ctrl + kBins, 3 * 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    ctx->st.launches++;
    static const int kG[3] = {8, 16, 32};
    for (int b = 0; b < 3; ++b) {
        const uint64_t nb = ctx->h_ctrl[kBins + b];
        if (!nb) continue;
        Window wb = w;
        wb.elist = bins + (size_t)b * w.W;
        wb.elist_n = (uint32_t)nb;
        wb.force_g = kG[b];
        TRY(extend_range(ctx, r, J, wb, 0, w.total, mode, nullptr, 0));
    }
    ctx->top = top_save;
    return CUTS_OK;
}

cuts_status alloc_window(cuts_ctx* ctx, int J, uint64_t W, Window* w) {
    size_t cub_bytes = 0;
    CK(cub::DeviceScan::ExclusiveSum(nullptr, cub_bytes, (uint64_t*)nullptr, (uint64_t*)nullptr, (int64_t)W + 1, ctx->stream));
    uint64_t off;
    TRY(alloc_top(ctx, window_scratch_bytes(W, J, cub_bytes), &off));
    char* p = ctx->arena + off;
    w->path = (uint32_t*)p; p += align_up((uint64_t)J * W * 4);
    w->src = (uint64_t*)p; p += align_up(W * 8);
    w->ub = (uint64_t*)p; p += align_up((W + 1) * 8);
    w->offs = (uint64_t*)p; p += align_up((W + 1) * 8);
    const uint64_t nl = (uint64_t)std::max(J - 1, 1);
    w->lst_off = (uint64_t*)p; p += align_up(nl * W * 8);
    w->lst_len = (uint32_t*)p; p += align_up(nl * W * 4);
    w->cpos = (uint64_t*)p; p += align_up((W + 1) * 8);
    w->cub_tmp = p;
    w->cub_bytes = cub_bytes;
    return CUTS_OK;
}

// window size for depth J: bounded so all depths' scratch takes <= 1/8 of the arena
uint64_t pick_window(cuts_ctx* ctx, uint64_t N) {
    uint64_t per = (uint64_t)(ctx->q.k) * 4 + 32 + (uint64_t)std::max<int>((int)ctx->q.k - 2, 1) * 12;   // path + src + ub + offs + cpos + list descriptors
    uint64_t budget = ctx->arena_bytes / 8 / std::max<uint32_t>(1, ctx->q.k - 1);
    uint64_t w = budget / per;
    w = std::max<uint64_t>(w, 1);
    w = std::min<uint64_t>(w, kMaxWindow);
    return std::min<uint64_t>(w, std::max<uint64_t>(N, 1));
}

void launch_export(cuts_ctx* ctx, int J, const Trie& t, uint64_t e0, uint64_t cnt, uint32_t* rows) {
    unsigned grid = (unsigned)std::min<uint64_t>((cnt + 255) / 256, (uint64_t)ctx->num_sms * 8);
    switch (J) {
        case 1: k_prefix_export<1><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
        case 2: k_prefix_export<2><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
        case 3: k_prefix_export<3><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
        case 4: k_prefix_export<4><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
        case 5: k_prefix_export<5><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
        case 6: k_prefix_export<6><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
        case 7: k_prefix_export<7><<<grid, 256, 0, ctx->stream>>>(t, e0, cnt, rows); break;
    }
}

// Dynamic redistribution (Alg. 3): at a chunk
// boundary ask the caller whether an idle peer wants work; if so give away the
// tail of the shallowest level that still has unplanned entries, exported as
// flat prefixes (reading P24), and shrink this context's range of that level.
cuts_status maybe_donate(cuts_ctx* ctx, Run& r) {
    if (!ctx->poll) return CUTS_OK;
    int d = 0;
    for (int j = 1; j < (int)ctx->q.k; ++j)
        if (ctx->dfs_on[j] && ctx->dfs_end[j] >= ctx->dfs_next[j] + 2) { d = j; break; }   // keep >= 1
    if (!d) return CUTS_OK;
    const uint64_t rem = ctx->dfs_end[d] - ctx->dfs_next[d];
    uint64_t give = std::min<uint64_t>(ctx->poll(ctx->user, (uint32_t)d, rem), rem);
    if (give == 0) return CUTS_OK;
    give = std::min<uint64_t>(give, free_bytes(ctx) / 2 / (4ull * d));
    if (give == 0) {   // no room to export: tell the caller (it may have claimed a receiver)
        if (ctx->ship(ctx->user, (uint32_t)d, nullptr, 0) != 0) return fail(ctx, CUTS_ECOMM, "donation ship callback failed");
        return CUTS_OK;
    }
    const uint64_t top_save = ctx->top;
    uint64_t off;
    TRY(alloc_top(ctx, give * 4ull * d, &off));
    uint32_t* rows = (uint32_t*)(ctx->arena + off);
    launch_export(ctx, d, r.t, ctx->dfs_end[d] - give, give, rows);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(ctx->stream));
    ctx->st.launches++;
    const int rc = ctx->ship(ctx->user, (uint32_t)d, rows, give);
    ctx->top = top_save;
    if (rc != 0) return fail(ctx, CUTS_ECOMM, "donation ship callback failed (%d)", rc);
    ctx->dfs_end[d] -= give;
    ctx->st.donated_entries += give;
    ctx->st.donations++;
    return CUTS_OK;
}

// HYBRID: process entries [0, N) of level J stored at r.t.lv[J] (DFS over chunks)
inline bool reuse_on(const cuts_ctx* ctx, const Run& r) {
    return r.mode == CUTS_HYBRID && !(ctx->debug & (CUTS_DEBUG_NO_REUSE | CUTS_DEBUG_SV));
}

// level J+1's chunk share of the free space: deeper stored levels (J+2 .. k-1)
// and their window scratch share the rest
cuts_status chunk_cap(cuts_ctx* ctx, int J, uint64_t* cap) {
    const int k = (int)ctx->q.k;
    uint64_t deeper_scratch = 0;
    const uint64_t wd = pick_window(ctx, ~0ull);
    size_t cb = 0;
    CK(cub::DeviceScan::ExclusiveSum(nullptr, cb, (uint64_t*)nullptr, (uint64_t*)nullptr, (int64_t)wd + 1, ctx->stream));
    for (int d = J + 1; d <= k - 1; ++d) deeper_scratch += window_scratch_bytes(wd, d, cb);
    const uint64_t fb = free_bytes(ctx);
    const uint64_t avail = fb > deeper_scratch ? fb - deeper_scratch : 0;
    const uint64_t share = avail / (uint64_t)(k - 1 - J);
    *cap = std::min<uint64_t>(share / sizeof(uint2), kMaxLevel);
    if (*cap == 0) return fail(ctx, CUTS_ENOMEM, "HYBRID: arena too small for level %d (free %llu B)", J + 1, (unsigned long long)fb);
    return CUTS_OK;
}

cuts_status hybrid_level(cuts_ctx* ctx, Run& r, int J, uint64_t N);

// unordered chunks over items [i0, i1) of window w (children bounded by ub)
cuts_status hybrid_items(cuts_ctx* ctx, Run& r, int J, const Window& w, uint64_t i0, uint64_t i1) {
    for (uint64_t t = i0; t < i1;) {
        uint64_t cap;
        TRY(chunk_cap(ctx, J, &cap));
        uint64_t t1 = std::min<uint64_t>(i1, t + cap);   // items bound children (ub)
        uint64_t off;
        const uint64_t bot_save = ctx->bot;
        TRY(alloc_bot(ctx, (t1 - t) * sizeof(uint2), &off));
        uint2* out = (uint2*)(ctx->arena + off);
        CK(cudaMemsetAsync(ctx->ctrl + kCursor, 0, sizeof(unsigned long long), ctx->stream));
        TRY(extend_range(ctx, r, J, w, t, t1, kWrite, out, t1 - t));
        CK(cudaMemcpyAsync(ctx->h_ctrl + kCursor, ctx->ctrl + kCursor, 8, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        uint64_t size = ctx->h_ctrl[kCursor];
        if (size > t1 - t) return fail(ctx, CUTS_ENOMEM, "internal: chunk overflow");
        ctx->st.level_size[J + 1] += size;
        ctx->bot = off + size * sizeof(uint2);     // shrink to the exact level size
        if (size) {
            r.t.lv[J + 1] = out;
            TRY(hybrid_level(ctx, r, J + 1, size));
        }
        ctx->bot = bot_save;
        t = t1;
        if (t < i1) TRY(maybe_donate(ctx, r));
    }
    return CUTS_OK;
}

// ordered chunks (level J+1 feeds an ancestor-set source deeper down): pass A
// counts each entry's children, a scan gives their exact offsets, chunks are cut
// at entry boundaries so each chunk holds whole sibling ranges, pass B writes
// every entry's children contiguously (no atomics).
cuts_status hybrid_ordered(cuts_ctx* ctx, Run& r, int J, Window& w) {
    CK(cudaMemsetAsync(w.ub, 0, (w.W + 1) * sizeof(uint64_t), ctx->stream));
    Window wa = w;
    wa.ord_cnt = w.ub;
    TRY(extend_range(ctx, r, J, wa, 0, w.total, kCount, nullptr, 0));
    if (ctx->debug & CUTS_DEBUG_GROUPS) {
        k_group_hist<<<std::min<uint32_t>((w.W + 255) / 256, 1024u), 256, 0, ctx->stream>>>(
            w.ub, w.W, ctx->ctrl + kGroupHist + 48 * (J + 1));
        CK(cudaGetLastError());
    }
    CK(cub::DeviceScan::ExclusiveSum(w.cub_tmp, w.cub_bytes, w.ub, w.cpos, (int64_t)w.W + 1, ctx->stream));
    ctx->st.launches += 2;
    for (uint32_t ea = 0; ea < w.W;) {
        uint64_t cap;
        TRY(chunk_cap(ctx, J, &cap));
        k_find_chunk<<<1, 1, 0, ctx->stream>>>(w.cpos, w.offs, w.W, ea, cap, ctx->ctrl + kFind);
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(ctx->h_ctrl + kFind, ctx->ctrl + kFind, 5 * 8, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        ctx->st.launches++;
        const uint32_t eb = (uint32_t)ctx->h_ctrl[kFind];
        const uint64_t size = ctx->h_ctrl[kFind + 1], i0 = ctx->h_ctrl[kFind + 2], i1 = ctx->h_ctrl[kFind + 3];
        if (eb > ea) {
            const uint64_t bot_save = ctx->bot;
            uint64_t off;
            TRY(alloc_bot(ctx, std::max<uint64_t>(size, 1) * sizeof(uint2), &off));
            uint2* out = (uint2*)(ctx->arena + off);
            if (size) {
                Window wb = w;
                wb.ord_pos = w.cpos;
                wb.ord_ea = ea;
                TRY(extend_range(ctx, r, J, wb, i0, i1, kWrite, out, size));
                ctx->st.level_size[J + 1] += size;
                ctx->ord[J] = {w.cpos, w.w0, ea, out, true, eb};
                r.t.lv[J + 1] = out;
                TRY(hybrid_level(ctx, r, J + 1, size));
                ctx->ord[J].valid = false;
            }
            ctx->bot = bot_save;
            ea = eb;
        } else {
            // one entry whose children exceed the share: unordered item pieces; its
            // subtree gets no ancestor-set source from level J
            TRY(hybrid_items(ctx, r, J, w, i0, ctx->h_ctrl[kFind + 4]));
            ea += 1;
        }
        if (ea < w.W) TRY(maybe_donate(ctx, r));
    }
    return CUTS_OK;
}

// symmetric last level (Reuse::sym conditions): is level J's count a pair count over
// sibling groups of the ordered level-(J-1) chunk?
bool sym_last(const cuts_ctx* ctx, const Run& r, int J) {
    const uint32_t a = ctx->anc[J];
    return J == (int)ctx->q.k - 1 && a && a + 1 == (uint32_t)J && reuse_on(ctx, r) && ctx->ord[a].valid &&
           !r.enumerate && !ctx->directed && (ctx->q.bw[J] & ~ctx->q.bw[a]) == (1u << a) && ctx->q.bwi[J] == 0 &&
           ctx->q.qdeg[J] <= ctx->q.qdeg[a] && !(ctx->debug & (CUTS_DEBUG_NO_PAIRS | CUTS_DEBUG_BINNED));
}

// local rows: level J = k-2 of a clique-like tail — the ordered level-J
// chunk's sibling groups carry both remaining extensions (J -> J+1 and the count)
bool lr_level(const cuts_ctx* ctx, const Run& r, int J) {
    const int k = (int)ctx->q.k;
    if (J != k - 2 || J < 3 || r.enumerate || ctx->directed || !reuse_on(ctx, r)) return false;
    if (ctx->debug & (CUTS_DEBUG_NO_PAIRS | CUTS_DEBUG_BINNED | CUTS_DEBUG_NO_LR)) return false;
    auto sym = [&](int L) {
        const uint32_t a = ctx->anc[L];
        return a && a + 1 == (uint32_t)L && (ctx->q.bw[L] & ~ctx->q.bw[a]) == (1u << a) && ctx->q.bwi[L] == 0 &&
               ctx->q.qdeg[L] <= ctx->q.qdeg[a];
    };
    return sym(J) && sym(J + 1) && ctx->ord[J - 1].valid;
}

// rows + bit algebra over the whole level-J chunk; returns the number of entries in
// groups too large for 64-bit rows (the windowed pipeline then takes those)
cuts_status lr_chunk(cuts_ctx* ctx, Run& r, int J, uint64_t N, uint64_t* large) {
    const auto& o = ctx->ord[J - 1];
    uint64_t off;
    TRY(alloc_top(ctx, N * 8, &off));
    unsigned long long* R = (unsigned long long*)(ctx->arena + off);
    CK(cudaMemsetAsync(R, 0, N * 8, ctx->stream));
    CK(cudaMemsetAsync(ctx->ctrl + kWork, 0, sizeof(unsigned long long), ctx->stream));
    CK(cudaMemsetAsync(ctx->ctrl + kLrLarge, 0, sizeof(unsigned long long), ctx->stream));
    const double m = (double)N / (double)std::max<uint64_t>(o.eb - o.ea, 1);
    const double avg = m / 2;
    const int cb = (ctx->debug & CUTS_DEBUG_BYTES) ? 1 : 0;
    int e0 = -1;
    if (ctx->debug & CUTS_DEBUG_TIMING) { e0 = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[e0], ctx->stream)); }
    auto go = [&](auto kern, int G) {
        static int occ[4] = {0, 0, 0, 0};
        int& oc = occ[cb ? 3 : (G == 8 ? 0 : (G == 16 ? 1 : 2))];
        if (!oc) { cudaOccupancyMaxActiveBlocksPerMultiprocessor(&oc, kern, 256, 0); if (oc < 1) oc = 1; }
        const uint64_t grid = std::min<uint64_t>((uint64_t)ctx->num_sms * oc, (N * G + 255) / 256 + 1);
        const uint32_t batch = (uint32_t)std::min(256.0, std::max(2.0, 2048.0 / std::max(avg, 1.0) / (32 / G)));
        kern<<<(unsigned)grid, 256, 0, ctx->stream>>>(r.g, r.t.lv[J], N, o.cpos, o.w0, o.ea, R, ctx->ctrl, batch);
    };
    if (cb) go(k_lr_rows<16, true>, 16);
    else if (avg >= 64) go(k_lr_rows<32, false>, 32);
    else if (avg >= 32) go(k_lr_rows<16, false>, 16);
    else go(k_lr_rows<8, false>, 8);
    CK(cudaGetLastError());
    const unsigned grid = (unsigned)std::min<uint64_t>((N + 255) / 256, (uint64_t)ctx->num_sms * 16);
    if (cb) k_lr_count<true><<<grid, 256, 0, ctx->stream>>>(r.g, r.t.lv[J], N, o.cpos, o.w0, o.ea, R, ctx->ctrl, r.t,
                                                           (uint32_t)J, ctx->q.bw[J], ctx->q.bw[J + 1]);
    else k_lr_count<false><<<grid, 256, 0, ctx->stream>>>(r.g, r.t.lv[J], N, o.cpos, o.w0, o.ea, R, ctx->ctrl, r.t,
                                                          (uint32_t)J, ctx->q.bw[J], ctx->q.bw[J + 1]);
    CK(cudaGetLastError());
    {   // mid-size groups: a CTA each, adjacency in shared memory
        static int occ = 0;
        if (!occ) { cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_lr_group<false>, 256, 0); if (occ < 1) occ = 1; }
        CK(cudaMemsetAsync(ctx->ctrl + kLrWork, 0, sizeof(unsigned long long), ctx->stream));
        auto kg = cb ? k_lr_group<true> : k_lr_group<false>;
        kg<<<(unsigned)(ctx->num_sms * occ), 256, 0, ctx->stream>>>(r.g, r.t.lv[J], o.cpos, o.ea, o.eb, ctx->ctrl, r.t,
                                                                    (uint32_t)J, ctx->q.bw[J], ctx->q.bw[J + 1]);
        CK(cudaGetLastError());
    }
    if (ctx->debug & CUTS_DEBUG_TIMING) {
        const int e1 = next_event(ctx);
        CK(cudaEventRecord(ctx->ev_pool[e1], ctx->stream));
        ctx->ev_ext.push_back({e0, e1});
    }
    CK(cudaMemcpyAsync(ctx->h_ctrl + kLrLarge, ctx->ctrl + kLrLarge, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    *large = ctx->h_ctrl[kLrLarge];
    ctx->st.chunks++;
    ctx->st.launches += 3;
    return CUTS_OK;
}

// deep local rows: level J = k-3 of a clique-like tail whose last three
// extensions only add adjacency to the newest vertex — the rows of the level-J sibling
// groups write level J+1 (stored, chunked) and carry levels J+2 and the count
bool dlr_level(const cuts_ctx* ctx, const Run& r, int J) {
    const int k = (int)ctx->q.k;
    if (J != k - 3 || J < 3 || r.enumerate || ctx->directed || !reuse_on(ctx, r)) return false;
    if (ctx->debug & (CUTS_DEBUG_NO_PAIRS | CUTS_DEBUG_BINNED | CUTS_DEBUG_NO_LR | CUTS_DEBUG_NO_DLR)) return false;
    auto sym = [&](int L) {
        const uint32_t a = ctx->anc[L];
        return a && a + 1 == (uint32_t)L && (ctx->q.bw[L] & ~ctx->q.bw[a]) == (1u << a) && ctx->q.bwi[L] == 0 &&
               ctx->q.qdeg[L] <= ctx->q.qdeg[a];
    };
    return sym(J) && sym(J + 1) && sym(J + 2) && ctx->ord[J - 1].valid;
}

// rows of the level-J chunk's groups, then level J+1 in entry-aligned chunks that fit
// the arena, each followed by the two-level tail; *large = entries left to the
// windowed pipeline (groups of more than kDlrMaxM members)
cuts_status dlr_chunk(cuts_ctx* ctx, Run& r, int J, uint64_t N, uint64_t* large, bool* applied) {
    const auto& o = ctx->ord[J - 1];
    const uint64_t ng = o.eb - o.ea;
    const int cb = (ctx->debug & CUTS_DEBUG_BYTES) ? 1 : 0;
    const bool timing = (ctx->debug & CUTS_DEBUG_TIMING) != 0;
    Dlr a{r.t.lv[J], N, o.cpos, o.w0, o.ea, o.eb, nullptr, nullptr, nullptr};
    size_t cub_bytes = 0;
    const uint64_t nscan = std::max<uint64_t>(ng, N) + 1;
    CK(cub::DeviceScan::ExclusiveSum(nullptr, cub_bytes, (uint64_t*)nullptr, (uint64_t*)nullptr, (int64_t)nscan, ctx->stream));
    uint64_t off;
    TRY(alloc_top(ctx, align_up((ng + 1) * 8) * 2 + align_up((N + 1) * 8) * 4 + align_up(cub_bytes), &off));
    char* p = ctx->arena + off;
    uint64_t* rw = (uint64_t*)p; p += align_up((ng + 1) * 8);
    uint64_t* roff = (uint64_t*)p; p += align_up((ng + 1) * 8);
    uint64_t* cnt = (uint64_t*)p; p += align_up((N + 1) * 8);
    uint64_t* cposb = (uint64_t*)p; p += align_up((N + 1) * 8);
    a.desc = (unsigned long long*)p; p += align_up((N + 1) * 8);
    uint64_t* cposn = (uint64_t*)p; p += align_up((N + 1) * 8);    // split layout: narrow entries' scan
    void* cub_tmp = p;
    int e0 = -1;
    if (timing) { e0 = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[e0], ctx->stream)); }
    CK(cudaMemsetAsync(ctx->ctrl + kDlrLarge, 0, 2 * sizeof(unsigned long long), ctx->stream));   // + kDlrWork
    const unsigned lg = (unsigned)std::min<uint64_t>((ng + 256) / 256, (uint64_t)ctx->num_sms * 8);
    k_dlr_layout<<<lg, 256, 0, ctx->stream>>>(a, rw, ctx->ctrl);
    CK(cudaGetLastError());
    CK(cub::DeviceScan::ExclusiveSum(cub_tmp, cub_bytes, rw, roff, (int64_t)ng + 1, ctx->stream));
    CK(cudaMemcpyAsync(ctx->h_ctrl + kDlrLarge, ctx->ctrl + kDlrLarge, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords + 8, roff + ng, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    *large = ctx->h_ctrl[kDlrLarge];
    const uint64_t words = ctx->h_ctrl[kCtrlWords + 8];
    // the rows must leave room for level-(J+1) chunks of a useful size; else the lr path
    *applied = words * 8 + (N + (1ull << 27)) * sizeof(uint2) <= free_bytes(ctx);
    if (!*applied) return CUTS_OK;
    TRY(alloc_top(ctx, std::max<uint64_t>(words, 1) * 8, &off));
    a.R = (unsigned long long*)(ctx->arena + off);
    a.roff = roff;
    CK(cudaMemsetAsync(a.R, 0, words * 8, ctx->stream));
    k_dlr_desc<<<(unsigned)std::min<uint64_t>((N + 255) / 256, (uint64_t)ctx->num_sms * 16), 256, 0, ctx->stream>>>(a);
    CK(cudaGetLastError());
    // the 129..1024-member groups, ascending by parent slot: k_dlr_tail_cta's work list
    const bool cta_tail = !cb && !(ctx->debug & (CUTS_DEBUG_TAIL_ALT | CUTS_DEBUG_TAIL_SPLIT | CUTS_DEBUG_NO_CTA_TAIL));
    DlrWide wide{nullptr, 0};
    if (cta_tail) {
        thrust::counting_iterator<uint32_t> it(0);
        const DlrIsWide pred{o.cpos, o.ea};
        size_t sel_bytes = 0;
        CK(cub::DeviceSelect::If(nullptr, sel_bytes, it, (uint32_t*)nullptr, ctx->ctrl + kNumSel, (int64_t)ng, pred, ctx->stream));
        uint64_t woff;
        TRY(alloc_top(ctx, align_up(std::max<uint64_t>(ng, 1) * 4) + align_up(sel_bytes), &woff));
        uint32_t* wl = (uint32_t*)(ctx->arena + woff);
        CK(cub::DeviceSelect::If(ctx->arena + woff + align_up(std::max<uint64_t>(ng, 1) * 4), sel_bytes, it, wl,
                                 ctx->ctrl + kNumSel, (int64_t)ng, pred, ctx->stream));
        CK(cudaMemcpyAsync(ctx->h_ctrl + kNumSel, ctx->ctrl + kNumSel, 8, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        wide = DlrWide{wl, (uint32_t)ctx->h_ctrl[kNumSel]};
    }
    // ... and the 2..64- and 65..128-member groups: k_dlr_tail_warp's work lists
    DlrWide narrow{nullptr, 0}, mid{nullptr, 0};
    if (cta_tail) {
        thrust::counting_iterator<uint32_t> it(0);
        const DlrIsMid pred{o.cpos, o.ea};
        size_t sel_bytes = 0;
        CK(cub::DeviceSelect::If(nullptr, sel_bytes, it, (uint32_t*)nullptr, ctx->ctrl + kNumSel, (int64_t)ng, pred, ctx->stream));
        uint64_t moff;
        TRY(alloc_top(ctx, align_up(std::max<uint64_t>(ng, 1) * 4) + align_up(sel_bytes), &moff));
        uint32_t* ml = (uint32_t*)(ctx->arena + moff);
        CK(cub::DeviceSelect::If(ctx->arena + moff + align_up(std::max<uint64_t>(ng, 1) * 4), sel_bytes, it, ml,
                                 ctx->ctrl + kNumSel, (int64_t)ng, pred, ctx->stream));
        CK(cudaMemcpyAsync(ctx->h_ctrl + kNumSel, ctx->ctrl + kNumSel, 8, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        mid = DlrWide{ml, (uint32_t)ctx->h_ctrl[kNumSel]};
    }
    if (cta_tail && (wide.n || mid.n)) {
        thrust::counting_iterator<uint32_t> it(0);
        const DlrIsNarrow pred{o.cpos, o.ea};
        size_t sel_bytes = 0;
        CK(cub::DeviceSelect::If(nullptr, sel_bytes, it, (uint32_t*)nullptr, ctx->ctrl + kNumSel, (int64_t)ng, pred, ctx->stream));
        uint64_t noff;
        TRY(alloc_top(ctx, align_up(std::max<uint64_t>(ng, 1) * 4) + align_up(sel_bytes), &noff));
        uint32_t* nl = (uint32_t*)(ctx->arena + noff);
        CK(cub::DeviceSelect::If(ctx->arena + noff + align_up(std::max<uint64_t>(ng, 1) * 4), sel_bytes, it, nl,
                                 ctx->ctrl + kNumSel, (int64_t)ng, pred, ctx->stream));
        CK(cudaMemcpyAsync(ctx->h_ctrl + kNumSel, ctx->ctrl + kNumSel, 8, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        narrow = DlrWide{nl, (uint32_t)ctx->h_ctrl[kNumSel]};
    }
    const double avg = (double)N / (double)std::max<uint64_t>(ng, 1) / 2;     // members tested per entry
    auto go = [&](auto kern, int G) {
        static int occ[4] = {0, 0, 0, 0};
        int& oc = occ[cb ? 3 : (G == 8 ? 0 : (G == 16 ? 1 : 2))];
        if (!oc) { cudaOccupancyMaxActiveBlocksPerMultiprocessor(&oc, kern, 256, 0); if (oc < 1) oc = 1; }
        const uint64_t grid = std::min<uint64_t>((uint64_t)ctx->num_sms * oc, (N * G + 255) / 256 + 1);
        const uint32_t batch = (uint32_t)std::min(256.0, std::max(2.0, 2048.0 / std::max(avg, 1.0) / (32 / G)));
        kern<<<(unsigned)grid, 256, 0, ctx->stream>>>(r.g, a, ctx->ctrl, batch);
    };
    if (cb) go(k_dlr_rows<16, true>, 16);
    else if (avg >= 64) go(k_dlr_rows<32, false>, 32);
    else if (avg >= 32) go(k_dlr_rows<16, false>, 16);   // C4 (avg 13): 8 lanes beat 16 (1.59 vs 1.64 s)
    else go(k_dlr_rows<8, false>, 8);
    CK(cudaGetLastError());
    const unsigned gc = (unsigned)std::min<uint64_t>((N + 256) / 256, (uint64_t)ctx->num_sms * 16);
    if (cb) k_dlr_counts<true><<<gc, 256, 0, ctx->stream>>>(r.g, r.t, a, cnt, ctx->ctrl, (uint32_t)J, ctx->q.bw[J]);
    else k_dlr_counts<false><<<gc, 256, 0, ctx->stream>>>(r.g, r.t, a, cnt, ctx->ctrl, (uint32_t)J, ctx->q.bw[J]);
    CK(cudaGetLastError());
    CK(cub::DeviceScan::ExclusiveSum(cub_tmp, cub_bytes, cnt, cposb, (int64_t)N + 1, ctx->stream));
    ctx->st.launches += 6;
    const bool split = wide.n > 0 || mid.n > 0;   // narrow children first, wide after (DlrOut)
    if (split) {
        k_dlr_narrow<<<gc, 256, 0, ctx->stream>>>(a, cnt, cnt);   // in place: cnt is not needed after the scan
        CK(cudaGetLastError());
        CK(cub::DeviceScan::ExclusiveSum(cub_tmp, cub_bytes, cnt, cposn, (int64_t)N + 1, ctx->stream));
        ctx->st.launches += 2;
    }
    if (timing) {
        const int e1 = next_event(ctx);
        CK(cudaEventRecord(ctx->ev_pool[e1], ctx->stream));
        ctx->ev_ext.push_back({e0, e1});
    }
    // level J+1 in entry-aligned chunks: write, then the two fused levels
    for (uint64_t ea = 0; ea < N;) {
        uint64_t cap;
        TRY(chunk_cap(ctx, J, &cap));
        k_find_chunk<<<1, 1, 0, ctx->stream>>>(cposb, cposb, (uint32_t)N, (uint32_t)ea, cap, ctx->ctrl + kFind);
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(ctx->h_ctrl + kFind, ctx->ctrl + kFind, 2 * 8, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        ctx->st.launches++;
        const uint64_t eb = ctx->h_ctrl[kFind], size = ctx->h_ctrl[kFind + 1];
        if (eb <= ea) return fail(ctx, CUTS_ENOMEM, "HYBRID: one level-%d entry's children exceed the arena share", J);
        uint32_t xa = 0, xb = 0;                  // parent slots of the chunk's first and last level-J entry
        uint64_t nn = 0;                          // split layout: narrow children in the chunk
        if (split && size) {
            CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords + 2, &a.lv[ea], 8, cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords + 3, &a.lv[eb - 1], 8, cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords + 4, cposn + ea, 8, cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords + 5, cposn + eb, 8, cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaStreamSynchronize(ctx->stream));
            xa = (uint32_t)((ctx->h_ctrl[kCtrlWords + 2] >> 32) - o.w0 - o.ea);
            xb = (uint32_t)((ctx->h_ctrl[kCtrlWords + 3] >> 32) - o.w0 - o.ea);
            nn = ctx->h_ctrl[kCtrlWords + 5] - ctx->h_ctrl[kCtrlWords + 4];
        }
        const DlrOut lay{cposb, split ? cposn : nullptr, ea, nn};
        if (size) {
            const uint64_t bot_save = ctx->bot;
            TRY(alloc_bot(ctx, size * sizeof(uint2), &off));
            uint2* out = (uint2*)(ctx->arena + off);
            int t0 = -1;
            if (timing) { t0 = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[t0], ctx->stream)); }
            const unsigned gw = (unsigned)std::min<uint64_t>((eb - ea + 15) / 16, (uint64_t)ctx->num_sms * 16);   // half-warp per entry
            k_dlr_write<<<gw, 256, 0, ctx->stream>>>(a, lay, eb, out);
            CK(cudaGetLastError());
            r.t.lv[J + 1] = out;
            int tm = -1;
            if (timing) { tm = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[tm], ctx->stream)); }
            const unsigned gt = (unsigned)std::min<uint64_t>((size + 255) / 256, (uint64_t)ctx->num_sms * 16);
            auto kt = cb ? k_dlr_tail<true, 0>
                          : ((ctx->debug & CUTS_DEBUG_TAIL_ALT) ? k_dlr_tail<false, 1>
                             : ((ctx->debug & CUTS_DEBUG_TAIL_SPLIT) ? k_dlr_tail<false, 2>
                                : k_dlr_tail<false, 0>));
            // split: the narrow-group entries [0, nn) with their own scan (k_dlr_tail reads
            // f - (cposn[e] - cposn[ea])); else the whole chunk with cposb
            if (split) {     // the narrow groups: a warp per group, rows in shared memory
                if (narrow.n && nn) {
                    CK(cudaMemsetAsync(ctx->ctrl + kDlrWork, 0, sizeof(unsigned long long), ctx->stream));
                    const unsigned gn = (unsigned)std::min<uint64_t>(((uint64_t)narrow.n + 63) / 64 + 1, (uint64_t)ctx->num_sms * 8);
                    k_dlr_tail_warp<1><<<gn, 256, 0, ctx->stream>>>(a, lay, eb, out, ctx->ctrl, narrow, xa, xb);
                    ctx->st.launches++;
                }
                if (mid.n) {
                    CK(cudaGetLastError());
                    CK(cudaMemsetAsync(ctx->ctrl + kDlrWork, 0, sizeof(unsigned long long), ctx->stream));
                    const unsigned gm = (unsigned)std::min<uint64_t>(((uint64_t)mid.n + 15) / 16 + 1, (uint64_t)ctx->num_sms * 8);
                    k_dlr_tail_warp<2><<<gm, 256, 0, ctx->stream>>>(a, lay, eb, out, ctx->ctrl, mid, xa, xb);
                    ctx->st.launches++;
                }
            } else {
                kt<<<gt, 256, 0, ctx->stream>>>(r.g, r.t, a, cposb, ea, out, size, ctx->ctrl,
                                                (uint32_t)(J + 1), ctx->q.bw[J + 1], ctx->q.bw[J + 2]);
            }
            CK(cudaGetLastError());
            if (wide.n) {   // the W >= 3 groups: a CTA per group, rows staged by TMA
                static int occ = 0;
                if (!occ) {
                    cudaFuncSetAttribute(k_dlr_tail_cta, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kDlrSmemBytes);
                    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_dlr_tail_cta, 256, kDlrSmemBytes);
                    if (occ < 1) occ = 1;
                }
                CK(cudaMemsetAsync(ctx->ctrl + kDlrWork, 0, sizeof(unsigned long long), ctx->stream));
                k_dlr_tail_cta<<<(unsigned)(ctx->num_sms * occ), 256, kDlrSmemBytes, ctx->stream>>>(
                    a, lay, eb, out, ctx->ctrl, wide, xa, xb);
                CK(cudaGetLastError());
                ctx->st.launches++;
            }
            CK(cudaGetLastError());
            if (timing) {
                const int t1 = next_event(ctx);
                CK(cudaEventRecord(ctx->ev_pool[t1], ctx->stream));
                ctx->ev_ext.push_back({t0, t1});
                ctx->ev_tail.push_back({tm, t1});
            }
            ctx->st.level_size[J + 1] += size;
            ctx->st.chunks++;
            ctx->st.launches += 2;
            ctx->bot = bot_save;
        }
        ea = eb;
    }
    return CUTS_OK;
}

// the whole level-J chunk in one k_pairs launch (no plan windows; with CUTS_DEBUG_BYTES
// the kernel also counts the §8.d model of its entries)
cuts_status pairs_level(cuts_ctx* ctx, Run& r, int J, uint64_t N) {
    const auto& o = ctx->ord[J - 1];
    const double m = (double)N / (double)std::max<uint64_t>(o.eb - o.ea, 1);   // siblings per group
    const double avg = m / 2;                                                  // tested per entry
    const int cb = (ctx->debug & CUTS_DEBUG_BYTES) ? 1 : 0;
    int e0 = -1;
    CK(cudaMemsetAsync(ctx->ctrl + kWork, 0, sizeof(unsigned long long), ctx->stream));
    if (ctx->debug & CUTS_DEBUG_TIMING) { e0 = next_event(ctx); CK(cudaEventRecord(ctx->ev_pool[e0], ctx->stream)); }
    auto go = [&](auto kern, int G) {
        static int occ[4] = {0, 0, 0, 0};
        int& oc = occ[cb ? 3 : (G == 8 ? 0 : (G == 16 ? 1 : 2))];
        if (!oc) { cudaOccupancyMaxActiveBlocksPerMultiprocessor(&oc, kern, 256, 0); if (oc < 1) oc = 1; }
        const uint64_t grid = std::min<uint64_t>((uint64_t)ctx->num_sms * oc, (N * G + 255) / 256 + 1);
        const uint32_t batch = (uint32_t)std::min(256.0, std::max(2.0, 2048.0 / std::max(avg, 1.0) / (32 / G)));
        kern<<<(unsigned)grid, 256, 0, ctx->stream>>>(r.g, r.t.lv[J], N, o.cpos, o.w0, o.ea, ctx->ctrl, batch,
                                                       r.t, (uint32_t)J, ctx->q.bw[J]);
    };
    if (cb) go(k_pairs<16, true>, 16);                   // instrumented (untimed) pass
    else if (avg >= 64) go(k_pairs<32, false>, 32);
    else if (avg >= 32) go(k_pairs<16, false>, 16);
    else go(k_pairs<8, false>, 8);
    CK(cudaGetLastError());
    if (ctx->debug & CUTS_DEBUG_TIMING) {
        const int e1 = next_event(ctx);
        CK(cudaEventRecord(ctx->ev_pool[e1], ctx->stream));
        ctx->ev_ext.push_back({e0, e1});
    }
    ctx->st.chunks++;
    ctx->st.launches += 2;
    return CUTS_OK;
}

cuts_status hybrid_level(cuts_ctx* ctx, Run& r, int J, uint64_t N) {
    const int k = (int)ctx->q.k;
    const bool last = (J == k - 1);
    const uint64_t top_save = ctx->top;
    if (last && sym_last(ctx, r, J)) return pairs_level(ctx, r, J, N);
    uint32_t skip_small = 0;
    bool dlr = false;
    if (dlr_level(ctx, r, J) && free_bytes(ctx) >= N * 40 + (64ull << 20)) {   // scans + descriptors + room
        uint64_t large = 0;
        TRY(dlr_chunk(ctx, r, J, N, &large, &dlr));
        ctx->top = top_save;
        if (dlr) {
            ctx->st.fused_levels |= 1ull << (J + 2);   // level k-1 of these groups is never stored
            if (large == 0) return CUTS_OK;
            skip_small = (uint32_t)kDlrMaxM;
        }
    }
    if (dlr) {
    } else if (lr_level(ctx, r, J) && free_bytes(ctx) >= N * 8 + (1u << 20)) {   // rows: 8 B per entry
        uint64_t large = 0;
        TRY(lr_chunk(ctx, r, J, N, &large));
        ctx->top = top_save;
        ctx->st.fused_levels |= 1ull << (J + 1);   // level k-1 of the small groups is never stored
        if (large == 0) return CUTS_OK;       // every group was small: nothing left at this level
        skip_small = (uint32_t)kLrMaxM;
    }
    const bool ordered = !last && reuse_on(ctx, r) && ((ctx->need_ord >> J) & 1u);
    ctx->dfs_on[J] = true;
    ctx->dfs_next[J] = 0;
    ctx->dfs_end[J] = N;
    for (uint64_t w0 = 0;;) {
        TRY(maybe_donate(ctx, r));
        N = ctx->dfs_end[J];          // a donation may have shrunk this level's range
        if (w0 >= N) break;
        Window w{};
        w.w0 = w0;
        w.W = (uint32_t)std::min<uint64_t>(pick_window(ctx, N), N - w0);
        ctx->dfs_next[J] = w0 + w.W;
        const uint32_t a = ctx->anc[J];
        if (a && reuse_on(ctx, r) && ctx->ord[a].valid)
            w.ru = Reuse{ctx->ord[a].lv, ctx->ord[a].cpos, ctx->ord[a].w0, ctx->ord[a].ea, a, ctx->q.bw[a],
                         sym_last(ctx, r, J) ? 1u : 0u, skip_small};
        TRY(alloc_window(ctx, J, w.W, &w));
        TRY(plan_window(ctx, r, J, w));
        if (last) {
            TRY(extend_last(ctx, r, J, w, r.enumerate ? kEnum : kCount));
        } else if (ordered) {
            TRY(hybrid_ordered(ctx, r, J, w));
        } else {
            TRY(hybrid_items(ctx, r, J, w, 0, w.total));
        }
        ctx->top = top_save;
        w0 += w.W;
    }
    ctx->dfs_on[J] = false;
    return CUTS_OK;
}

// BFS: every level stored whole (Alg. 1); ENOMEM when a level does not fit
cuts_status bfs_levels(cuts_ctx* ctx, Run& r, int J0, uint64_t N1, int jstop = 0) {
    const int k = (int)ctx->q.k;
    uint64_t N = N1;
    const int jend = jstop ? jstop : k;           // extend J -> J+1 while J < jend
    for (int J = J0; J < jend && J <= k - 1 && N > 0; ++J) {
        const bool last = (J == k - 1);
        const uint64_t top_save = ctx->top;
        uint64_t W = pick_window(ctx, N);
        Window w{};
        TRY(alloc_window(ctx, J, W, &w));
        uint2* out = nullptr;
        uint64_t cap = 0, off = 0;
        if (!last) {
            cap = std::min<uint64_t>(free_bytes(ctx) / sizeof(uint2), kMaxLevel);
            if (cap == 0) return fail(ctx, CUTS_ENOMEM, "BFS: no room for level %d", J + 1);
            TRY(alloc_bot(ctx, cap * sizeof(uint2), &off));
            out = (uint2*)(ctx->arena + off);
            CK(cudaMemsetAsync(ctx->ctrl + kCursor, 0, sizeof(unsigned long long), ctx->stream));
        }
        uint64_t run = 0;                   // jstop: entries written so far (ordered levels)
        for (uint64_t w0 = 0; w0 < N; w0 += W) {
            w.w0 = w0;
            w.W = (uint32_t)std::min<uint64_t>(W, N - w0);
            TRY(plan_window(ctx, r, J, w));
            if (last) TRY(extend_last(ctx, r, J, w, r.enumerate ? kEnum : kCount));
            else if (jstop) {
                // the partition prefix (cuts_set_partition_depth) must be the same list on
                // every part: write it ORDERED (per-entry counts, scan, children at exact
                // offsets in candidate order) instead of by warp-aggregated atomics
                CK(cudaMemsetAsync(w.ub, 0, (w.W + 1) * sizeof(uint64_t), ctx->stream));
                Window wa = w;
                wa.ord_cnt = w.ub;
                TRY(extend_range(ctx, r, J, wa, 0, w.total, kCount, nullptr, 0));
                CK(cub::DeviceScan::ExclusiveSum(w.cub_tmp, w.cub_bytes, w.ub, w.cpos, (int64_t)w.W + 1, ctx->stream));
                CK(cudaMemcpyAsync(ctx->h_ctrl + kCtrlWords + 1, w.cpos + w.W, 8, cudaMemcpyDeviceToHost, ctx->stream));
                CK(cudaStreamSynchronize(ctx->stream));
                const uint64_t sz = ctx->h_ctrl[kCtrlWords + 1];
                if (run + sz > cap)
                    return fail(ctx, CUTS_ENOMEM, "partition prefix: level %d does not fit the arena", J + 1);
                Window wb = w;
                wb.ord_pos = w.cpos;
                wb.ord_ea = 0;
                TRY(extend_range(ctx, r, J, wb, 0, w.total, kWrite, out + run, sz));
                run += sz;
                ctx->h_ctrl[kCursor] = run;
                CK(cudaMemcpyAsync(ctx->ctrl + kCursor, ctx->h_ctrl + kCursor, 8, cudaMemcpyHostToDevice, ctx->stream));
                continue;
            }
            else TRY(extend_range(ctx, r, J, w, 0, w.total, kWrite, out, cap));
            if (!last && w0 + W < N) {     // stop at the first window that overflows the level
                CK(cudaMemcpyAsync(ctx->h_ctrl + kCursor, ctx->ctrl + kCursor, 8, cudaMemcpyDeviceToHost, ctx->stream));
                CK(cudaStreamSynchronize(ctx->stream));
                if (ctx->h_ctrl[kCursor] > cap)
                    return fail(ctx, CUTS_ENOMEM, "BFS: level %d exceeds the room for %llu entries after %llu of %llu "
                                "entries of level %d (use CUTS_HYBRID)", J + 1, (unsigned long long)cap,
                                (unsigned long long)(w0 + W), (unsigned long long)N, J);
            }
        }
        if (!last) {
            CK(cudaMemcpyAsync(ctx->h_ctrl + kCursor, ctx->ctrl + kCursor, 8, cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaStreamSynchronize(ctx->stream));
            uint64_t size = ctx->h_ctrl[kCursor];
            ctx->st.level_size[J + 1] = size;
            if (size > cap)
                return fail(ctx, CUTS_ENOMEM, "BFS: level %d has %llu entries, room for %llu (use CUTS_HYBRID)", J + 1,
                            (unsigned long long)size, (unsigned long long)cap);
            ctx->bot = off + size * sizeof(uint2);
            r.t.lv[J + 1] = out;
            N = size;
        }
        ctx->top = top_save;
    }
    return CUTS_OK;
}

// hub bitmaps (SV-style membership rows) after deg; moves base_off
cuts_status build_hubs(cuts_ctx* ctx) {
    ctx->nhubs = 0;
    ctx->hub_t_used = 0;
    ctx->hub = nullptr;
    ctx->bm = nullptr;
    ctx->cb = nullptr;
    if (ctx->hub_t == 0xFFFFFFFFu || ctx->n == 0 || ctx->nnz == 0) return CUTS_OK;
    const uint32_t n = ctx->n;
    ctx->words = (n + 31) / 32;
    const uint64_t row_bytes = (uint64_t)ctx->words * 4;
    const uint64_t budget = std::min<uint64_t>(ctx->arena_bytes / 16, 8ull << 30);
    unsigned grid = (unsigned)std::min<uint64_t>(((uint64_t)n + 255) / 256, (uint64_t)ctx->num_sms * 8);
    uint32_t t = ctx->hub_t;
    CK(cudaMemsetAsync(ctx->ctrl, 0, kCtrlWords * sizeof(unsigned long long), ctx->stream));
    if (t == 0) {   // automatic: smallest power of two >= 256 whose rows fit the budget
        k_hub_hist<<<grid, 256, 0, ctx->stream>>>(ctx->deg, n, ctx->ctrl + 16);
        CK(cudaGetLastError());
        TRY(read_ctrl(ctx));
        t = 0;
        for (int b = 8; b < 32; ++b) {
            uint64_t cnt = 0;
            for (int b2 = b; b2 < 32; ++b2) cnt += ctx->h_ctrl[16 + b2];
            if (cnt * row_bytes <= budget) { t = 1u << b; break; }
        }
        if (t == 0) return CUTS_OK;
        CK(cudaMemsetAsync(ctx->ctrl, 0, kCtrlWords * sizeof(unsigned long long), ctx->stream));
    }
    const uint64_t hub_bytes = align_up((uint64_t)n * 4);
    if (ctx->base_off + hub_bytes + (64u << 10) > ctx->arena_bytes) return CUTS_OK;   // no room: skip
    ctx->hub = (uint32_t*)(ctx->arena + ctx->base_off);
    k_hub_mark<<<grid, 256, 0, ctx->stream>>>(ctx->deg, n, t, ctx->hub, ctx->ctrl + kNumSel);
    CK(cudaGetLastError());
    TRY(read_ctrl(ctx));
    const uint64_t nh = ctx->h_ctrl[kNumSel];
    const uint64_t bm_bytes = align_up(nh * row_bytes);
    if (nh == 0 || ctx->base_off + hub_bytes + bm_bytes + (64u << 10) > ctx->arena_bytes) {
        ctx->hub = nullptr;
        return CUTS_OK;   // nothing to do, or does not fit: binary search everywhere
    }
    ctx->bm = (uint32_t*)(ctx->arena + ctx->base_off + hub_bytes);
    CK(cudaMemsetAsync(ctx->bm, 0, nh * row_bytes, ctx->stream));
    // core bitmap: hub x hub adjacency in hub-row coordinates, when it is small (<= 64 MB)
    ctx->cb = nullptr;
    ctx->cbw = (uint32_t)((nh + 31) / 32);
    const uint64_t cb_bytes = align_up(nh * (uint64_t)ctx->cbw * 4);
    if (cb_bytes <= (64ull << 20) && ctx->base_off + hub_bytes + bm_bytes + cb_bytes + (64u << 10) <= ctx->arena_bytes) {
        ctx->cb = (uint32_t*)(ctx->arena + ctx->base_off + hub_bytes + bm_bytes);
        CK(cudaMemsetAsync(ctx->cb, 0, cb_bytes, ctx->stream));
    }
    unsigned g2 = (unsigned)std::min<uint64_t>(((uint64_t)n * 32 + 255) / 256, (uint64_t)ctx->num_sms * 16);
    k_hub_fill<<<g2, 256, 0, ctx->stream>>>(ctx->row_ptr, ctx->col, n, ctx->hub, ctx->words, ctx->bm, ctx->cb, ctx->cbw);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(ctx->stream));
    ctx->nhubs = nh;
    ctx->hub_t_used = t;
    ctx->base_off += hub_bytes + bm_bytes + (ctx->cb ? cb_bytes : 0);
    return CUTS_OK;
}

// canonical level-1 list {u : deg(u) >= deg_Q(S[0])} in ascending id (CUB select
// over a counting iterator), cached per (graph, query): every root chunk of the
// multi-GPU queue reuses it instead of re-running the O(n) select
cuts_status ensure_canonical(cuts_ctx* ctx) {
    if (ctx->canon_valid) return CUTS_OK;
    ctx->bot = ctx->base_off;
    ctx->top = ctx->arena_bytes & ~(kAlign - 1);
    uint64_t off_canon, off_tmp;
    TRY(alloc_bot(ctx, (uint64_t)ctx->n * 4 + 4, &off_canon));
    uint32_t* canon = (uint32_t*)(ctx->arena + off_canon);
    DegAtLeast pred{ctx->deg, ctx->q.qdeg[0], ctx->directed ? ctx->n : 0u, ctx->q.qdin[0]};
    thrust::counting_iterator<uint32_t> it(0);
    size_t tmp_bytes = 0;
    unsigned long long* d_num = ctx->ctrl + kNumSel;
    CK(cub::DeviceSelect::If(nullptr, tmp_bytes, it, canon, d_num, (int64_t)ctx->n, pred, ctx->stream));
    TRY(alloc_top(ctx, tmp_bytes, &off_tmp));
    CK(cub::DeviceSelect::If(ctx->arena + off_tmp, tmp_bytes, it, canon, d_num, (int64_t)ctx->n, pred, ctx->stream));
    TRY(read_ctrl(ctx));
    ctx->canon = canon;
    ctx->canon_n = ctx->h_ctrl[kNumSel];
    ctx->run_off = align_up(off_canon + ctx->canon_n * 4 + 4);
    ctx->canon_valid = true;
    return CUTS_OK;
}

// level 1: canonical list -> root range -> shuffle -> slice
// seeded Feistel bijection of [0, R) (reading P25)
Shuffle make_shuffle(uint64_t seed, uint64_t R) {
    Shuffle sh{};
    sh.R = R;
    uint32_t bits = 2;
    while ((1ull << bits) < R) ++bits;
    if (bits & 1) ++bits;
    sh.half = bits / 2;
    sh.mask = (uint32_t)((1ull << sh.half) - 1);
    uint64_t x = seed;
    for (int i = 0; i < 4; ++i) {   // splitmix64 round keys
        x += 0x9E3779B97F4A7C15ull;
        uint64_t z = x;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        sh.key[i] = z ^ (z >> 31);
    }
    return sh;
}

// positions [sb, se) of a list of R with p % nparts == part: first position, count
void slice_of(const cuts_ctx* ctx, uint64_t R, uint64_t* p0, uint64_t* cnt) {
    const uint64_t sb = std::min(ctx->slice_begin, R), se = std::min(ctx->slice_end, R);
    *p0 = 0;
    *cnt = 0;
    if (se > sb) {
        *p0 = sb + ((ctx->part + ctx->nparts - (uint32_t)(sb % ctx->nparts)) % ctx->nparts);
        *cnt = *p0 < se ? (se - *p0 + ctx->nparts - 1) / ctx->nparts : 0;
    }
}

cuts_status build_level1(cuts_ctx* ctx, Run& r, uint64_t* n1) {
    const uint32_t* canon = ctx->canon;
    const uint64_t ncanon = ctx->canon_n;
    ctx->st.level1_canonical = ncanon;
    uint64_t rb = std::min(ctx->root_begin, ncanon), re = std::min(ctx->root_end, ncanon);
    if (re < rb) re = rb;
    const uint64_t R = re - rb;
    // slice of shuffled positions [sb, se) with p % nparts == part
    uint64_t cnt = 0, p0 = 0;
    slice_of(ctx, R, &p0, &cnt);
    uint64_t off_l1;
    TRY(alloc_bot(ctx, std::max<uint64_t>(cnt, 1) * sizeof(uint2), &off_l1));
    uint2* L1 = (uint2*)(ctx->arena + off_l1);
    if (cnt) {
        const Shuffle sh = make_shuffle(ctx->seed, R);
        unsigned grid = (unsigned)std::min<uint64_t>((cnt + 255) / 256, (uint64_t)ctx->num_sms * 8);
        k_level1<<<grid, 256, 0, ctx->stream>>>(canon, rb, sh, p0, ctx->nparts, cnt, L1);
        CK(cudaGetLastError());
        ctx->st.launches++;
    }
    r.t.lv[1] = L1;
    *n1 = cnt;
    return CUTS_OK;
}

// component roots (bw[J] == 0, J > 0): their candidate set is the
// cross-product factor {v : deg(v) >= qdeg[J]}, ascending, built once per run
// on the bottom stack (the extend kernel reads it like a CSR source list)
cuts_status build_free_lists(cuts_ctx* ctx, Run& r) {
    r.g.fre = (const uint32_t*)ctx->arena;
    int roots = 0;
    for (uint32_t J = 1; J < ctx->q.k; ++J) roots += (ctx->q.bw[J] | ctx->q.bwi[J]) ? 0 : 1;
    // the lists take n u32 each: when they would crowd the trie (more than 1/8 of the
    // free arena), a component root streams the identity list [0, n) instead and the
    // extend kernel applies its degree filter (same candidates, no memory)
    const bool identity = roots && (uint64_t)roots * ((uint64_t)ctx->n * 4 + 4 + kAlign) > free_bytes(ctx) / 8;
    for (uint32_t J = 1; J < ctx->q.k; ++J) {
        ctx->q.foff[J] = 0;
        ctx->q.flen[J] = 0;
        if (ctx->q.bw[J] | ctx->q.bwi[J]) continue;
        if (identity) {
            ctx->q.foff[J] = kIdSrc;
            ctx->q.flen[J] = ctx->n;
            continue;
        }
        uint64_t off_list;
        TRY(alloc_bot(ctx, (uint64_t)ctx->n * 4 + 4, &off_list));
        const uint64_t top_save = ctx->top;
        DegAtLeast pred{ctx->deg, ctx->q.qdeg[J], ctx->directed ? ctx->n : 0u, ctx->q.qdin[J]};
        thrust::counting_iterator<uint32_t> it(0);
        size_t tmp_bytes = 0;
        uint64_t off_tmp;
        uint32_t* list = (uint32_t*)(ctx->arena + off_list);
        CK(cub::DeviceSelect::If(nullptr, tmp_bytes, it, list, ctx->ctrl + kNumSel, (int64_t)ctx->n, pred, ctx->stream));
        TRY(alloc_top(ctx, tmp_bytes, &off_tmp));
        CK(cub::DeviceSelect::If(ctx->arena + off_tmp, tmp_bytes, it, list, ctx->ctrl + kNumSel, (int64_t)ctx->n, pred,
                                 ctx->stream));
        TRY(read_ctrl(ctx));
        ctx->top = top_save;
        ctx->q.foff[J] = off_list / 4;
        ctx->q.flen[J] = (uint32_t)ctx->h_ctrl[kNumSel];
        ctx->st.launches += 2;
    }
    ctx->st.free_identity = identity ? 1 : 0;
    return CUTS_OK;
}

// flat-prefix seeding: levels 1..pre_j as a chain trie over the caller's rows
cuts_status build_prefix_levels(cuts_ctx* ctx, Run& r, uint32_t J, uint64_t cnt, const uint32_t* rows) {
    for (uint32_t l = 1; l <= J; ++l) {
        uint64_t off;
        TRY(alloc_bot(ctx, std::max<uint64_t>(cnt, 1) * sizeof(uint2), &off));
        r.t.lv[l] = (uint2*)(ctx->arena + off);
        ctx->st.level_size[l] = cnt;
    }
    if (cnt) {
        unsigned grid = (unsigned)std::min<uint64_t>((cnt + 255) / 256, (uint64_t)ctx->num_sms * 8);
        k_prefix_import<<<grid, 256, 0, ctx->stream>>>(rows, J, cnt, r.t);
        CK(cudaGetLastError());
        ctx->st.launches++;
    }
    return CUTS_OK;
}

// cuts_set_partition_depth D > 1: levels 1..D are built whole (BFS over the root range,
// the same on every part), the seeded shuffle of level D is sliced like the level-1 list
// (P:1277-1279 one level down) and the slice is extended from flat prefixes.  Levels
// below D are reported only by the part holding shuffled position 0 (part 0 of the slice
// that starts at 0), so summing the stats of all parts gives the exact level sizes.
cuts_status partition_run(cuts_ctx* ctx, Run& r, cuts_mode mode) {
    const int D = (int)ctx->part_depth;
    const uint64_t sb0 = ctx->slice_begin, se0 = ctx->slice_end;
    const uint32_t pt = ctx->part, np = ctx->nparts;
    ctx->slice_begin = 0;
    ctx->slice_end = ~0ull;
    ctx->part = 0;
    ctx->nparts = 1;
    uint64_t n1 = 0;
    const cuts_status s1 = build_level1(ctx, r, &n1);
    ctx->slice_begin = sb0;
    ctx->slice_end = se0;
    ctx->part = pt;
    ctx->nparts = np;
    TRY(s1);
    ctx->st.level_size[1] = n1;
    if (n1) TRY(bfs_levels(ctx, r, 1, n1, D));
    const uint64_t ND = ctx->st.level_size[D];
    if (ctx->size_only) return read_ctrl(ctx);
    uint64_t p0 = 0, cnt = 0;
    slice_of(ctx, ND, &p0, &cnt);
    uint64_t off;
    TRY(alloc_bot(ctx, std::max<uint64_t>(cnt * D, 1) * sizeof(uint32_t), &off));
    uint32_t* prows = (uint32_t*)(ctx->arena + off);
    if (cnt) {
        const Shuffle sh = make_shuffle(ctx->seed, ND);
        const unsigned grid = (unsigned)std::min<uint64_t>((cnt + 255) / 256, (uint64_t)ctx->num_sms * 8);
        switch (D) {
            case 2: k_prefix_slice<2><<<grid, 256, 0, ctx->stream>>>(r.t, sh, p0, np, cnt, prows); break;
            case 3: k_prefix_slice<3><<<grid, 256, 0, ctx->stream>>>(r.t, sh, p0, np, cnt, prows); break;
            case 4: k_prefix_slice<4><<<grid, 256, 0, ctx->stream>>>(r.t, sh, p0, np, cnt, prows); break;
            case 5: k_prefix_slice<5><<<grid, 256, 0, ctx->stream>>>(r.t, sh, p0, np, cnt, prows); break;
            case 6: k_prefix_slice<6><<<grid, 256, 0, ctx->stream>>>(r.t, sh, p0, np, cnt, prows); break;
            default: k_prefix_slice<7><<<grid, 256, 0, ctx->stream>>>(r.t, sh, p0, np, cnt, prows); break;
        }
        CK(cudaGetLastError());
        ctx->st.launches++;
    }
    uint64_t upper[kMaxK + 1];
    const bool first = std::min(sb0, ND) == 0 && pt == 0;
    for (int l = 0; l <= kMaxK; ++l) upper[l] = (first && l < D) ? ctx->st.level_size[l] : 0;
    TRY(build_prefix_levels(ctx, r, (uint32_t)D, cnt, prows));
    for (int l = 1; l < D; ++l) ctx->st.level_size[l] = upper[l];
    ctx->st.level_size[D] = cnt;
    if (cnt) {
        if (mode == CUTS_BFS) TRY(bfs_levels(ctx, r, D, cnt));
        else TRY(hybrid_level(ctx, r, D, cnt));
    }
    return read_ctrl(ctx);
}

cuts_status run_query(cuts_ctx* ctx, cuts_mode mode, bool enumerate, uint32_t* rows, uint64_t cap_rows) {
    if (!ctx) return CUTS_EINVAL;
    if (!ctx->has_graph || !ctx->has_query) return fail(ctx, CUTS_ESTATE, "load_graph and set_query must precede count/enumerate");
    if (mode != CUTS_BFS && mode != CUTS_HYBRID) return fail(ctx, CUTS_EINVAL, "bad mode %d", (int)mode);
    if (enumerate && !rows && cap_rows) return fail(ctx, CUTS_EINVAL, "null d_out with cap_rows > 0");
    auto t_start = std::chrono::steady_clock::now();
    CK(cudaSetDevice(ctx->device));
    ctx->st = cuts_stats{};
    ctx->st.k = ctx->q.k;
    for (uint32_t i = 0; i < ctx->q.k; ++i) ctx->st.order[i] = ctx->q.S[i];
    ctx->ev_used = 0;
    ctx->ev_ext.clear();
    ctx->ev_tail.clear();
    ctx->ev_plan.clear();
    if (!ctx->pre_j) TRY(ensure_canonical(ctx));
    ctx->bot = ctx->canon_valid ? ctx->run_off : ctx->base_off;
    ctx->top = ctx->arena_bytes & ~(kAlign - 1);
    ctx->peak = ctx->bot;
    CK(cudaMemsetAsync(ctx->ctrl, 0, kCtrlWords * sizeof(unsigned long long), ctx->stream));
    if (ctx->debug & CUTS_DEBUG_GROUPS)
        CK(cudaMemsetAsync(ctx->ctrl + kGroupHist, 0, kGroupHistWords * sizeof(unsigned long long), ctx->stream));
    if (ctx->debug & CUTS_DEBUG_PRELOAD_COUNT) {   // test hook: the 128-bit carry and CUTS_EOVERFLOW
        ctx->h_ctrl[kCtrlWords + 16] = kPreloadCount;
        CK(cudaMemcpyAsync(ctx->ctrl + kCountLo, ctx->h_ctrl + kCtrlWords + 16, 8, cudaMemcpyHostToDevice, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
    }

    Run r{};
    r.mode = mode;
    r.enumerate = enumerate;
    r.rows = rows;
    r.cap_rows = cap_rows;
    if (ctx->q_directed != ctx->directed)
        return fail(ctx, CUTS_EINVAL, "%s query on a %s graph", ctx->q_directed ? "directed" : "undirected",
                    ctx->directed ? "directed" : "undirected");
    r.g = Graph{ctx->row_ptr, ctx->col, ctx->deg, ctx->nhubs ? ctx->hub : nullptr, ctx->bm, ctx->n, ctx->words, ctx->colx};
    if (ctx->nhubs && ctx->cb) { r.g.cb = ctx->cb; r.g.cbw = ctx->cbw; }
    r.g.dn = ctx->directed ? ctx->n : 0u;
    ctx->q.src_first = (ctx->debug & CUTS_DEBUG_FIRST_SOURCE) ? 1u : 0u;
    ctx->q.count_fast = (!enumerate && !(ctx->debug & (CUTS_DEBUG_NO_FAST_COUNT | CUTS_DEBUG_SV))) ? 1u : 0u;
    ctx->sv = nullptr;
    ctx->sv_warps = 0;
    if (ctx->debug & CUTS_DEBUG_SV) {   // ablation: per-warp scatter vectors, CSR lists only
        if (ctx->directed) return fail(ctx, CUTS_EUNSUPPORTED, "CUTS_DEBUG_SV is undirected only");
        r.g.hub = nullptr;
        uint64_t warps = (uint64_t)ctx->num_sms * 16;
        const uint64_t room = free_bytes(ctx) / 4;
        while (warps > 8 && warps * ctx->n > room) warps /= 2;
        uint64_t off;
        TRY(alloc_bot(ctx, warps * ctx->n + 16, &off));
        ctx->sv = (uint8_t*)(ctx->arena + off);
        ctx->sv_warps = warps & ~7ull;
        CK(cudaMemsetAsync(ctx->sv, 0, warps * ctx->n, ctx->stream));
    }
    TRY(build_free_lists(ctx, r));
    uint64_t n1 = 0;
    const int k = (int)ctx->q.k;
    for (int j = 0; j <= kMaxK; ++j) { ctx->dfs_on[j] = false; ctx->dfs_next[j] = ctx->dfs_end[j] = 0; ctx->ord[j].valid = false; }
    if (ctx->pre_j) {
        TRY(build_prefix_levels(ctx, r, ctx->pre_j, ctx->pre_count, ctx->pre_rows));
        const int J0 = (int)ctx->pre_j;
        if (ctx->pre_count > 0) {
            if (mode == CUTS_BFS) TRY(bfs_levels(ctx, r, J0, ctx->pre_count));
            else TRY(hybrid_level(ctx, r, J0, ctx->pre_count));
        }
        TRY(read_ctrl(ctx));
    } else if (ctx->part_depth > 1 && (int)ctx->part_depth < k) {
        TRY(partition_run(ctx, r, mode));
    } else {
    TRY(build_level1(ctx, r, &n1));
    ctx->st.level_size[1] = n1;
    if (k == 1) {
        if (enumerate && n1 && cap_rows) {
            unsigned grid = (unsigned)std::min<uint64_t>((n1 + 255) / 256, (uint64_t)ctx->num_sms * 8);
            k_rows_k1<<<grid, 256, 0, ctx->stream>>>(r.t.lv[1], n1, rows, cap_rows);
            CK(cudaGetLastError());
        }
        ctx->h_ctrl[kCountLo] = n1;
        ctx->h_ctrl[kCountHi] = 0;
        ctx->h_ctrl[kEnumCursor] = n1;
        CK(cudaStreamSynchronize(ctx->stream));
    } else if (n1 > 0) {
        if (mode == CUTS_BFS) TRY(bfs_levels(ctx, r, 1, n1));
        else TRY(hybrid_level(ctx, r, 1, n1));
        TRY(read_ctrl(ctx));
    } else {
        TRY(read_ctrl(ctx));
    }
    }
    if (enumerate) {
        ctx->st.count_lo = ctx->h_ctrl[kEnumCursor];
        ctx->st.count_hi = 0;
    } else {
        ctx->st.count_lo = ctx->h_ctrl[kCountLo];
        ctx->st.count_hi = ctx->h_ctrl[kCountHi];
    }
    if (ctx->h_ctrl[kErr]) return fail(ctx, CUTS_ECUDA, "internal: %llu deep-rows tail entries out of range",
                                       (unsigned long long)ctx->h_ctrl[kErr]);
    if (k > 1) ctx->st.level_size[k] = ctx->st.count_lo;
    if (k >= 5) ctx->st.level_size[k - 1] += ctx->h_ctrl[kLrLevel];   // local rows: |L_{k-1}| of the small groups
    ctx->st.alg_bytes_plan = ctx->h_ctrl[kBytesPlan];
    ctx->st.alg_bytes_extend = ctx->h_ctrl[kBytesExt] + ctx->h_ctrl[kBytesOut];
    ctx->st.alg_bytes_extend_needed = ctx->h_ctrl[kBytesNeed] + ctx->h_ctrl[kBytesOut];
    ctx->st.peak_arena_bytes = ctx->peak;
    ctx->st.hubs = ctx->nhubs;
    ctx->st.hub_threshold = ctx->hub_t_used;
    if (ctx->debug & CUTS_DEBUG_TIMING) {
        double ms = 0;
        for (auto& pr : ctx->ev_ext) {
            float f = 0;
            CK(cudaEventElapsedTime(&f, ctx->ev_pool[pr.first], ctx->ev_pool[pr.second]));
            ms += f;
        }
        ctx->st.ms_extend = ms;
        ctx->st.extend_launches = ctx->ev_ext.size();
        ms = 0;
        for (auto& pr : ctx->ev_plan) {
            float f = 0;
            CK(cudaEventElapsedTime(&f, ctx->ev_pool[pr.first], ctx->ev_pool[pr.second]));
            ms += f;
        }
        ctx->st.ms_plan = ms;
        ms = 0;
        for (auto& pr : ctx->ev_tail) {
            float f = 0;
            CK(cudaEventElapsedTime(&f, ctx->ev_pool[pr.first], ctx->ev_pool[pr.second]));
            ms += f;
        }
        ctx->st.ms_tail = ms;
        ctx->st.tail_launches = ctx->ev_tail.size();
    }
    ctx->st.tail_word_ops = ctx->h_ctrl[kTailOps];
    ctx->st.ms_total = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count();
    return CUTS_OK;
}

}  // namespace

namespace {
cuts_status finish_query(cuts_ctx* ctx, const QPlan& qp, bool directed) {
    ctx->q = qp;
    ctx->q_directed = directed;
    ctx->canon_valid = false;
    // ancestor-set reuse plan: deepest a in [2, J-1] with |bw[a]| >= 2 (an actual
    // intersection), bw[a] a subset of bw[J] and deg_Q(S[a]) <= deg_Q(S[J])
    // (undirected only)
    ctx->need_ord = 0;
    for (uint32_t J = 0; J <= kMaxK; ++J) ctx->anc[J] = 0;
    for (uint32_t J = 3; J < qp.k && !directed; ++J)
        for (uint32_t a = J - 1; a >= 2; --a)
            if (__builtin_popcount(qp.bw[a]) >= 2 && (qp.bw[a] & ~qp.bw[J]) == 0 && qp.qdeg[a] <= qp.qdeg[J]) {
                ctx->anc[J] = a;
                ctx->need_ord |= 1u << a;
                break;
            }
    ctx->root_begin = 0;
    ctx->root_end = ~0ull;
    ctx->slice_begin = 0;
    ctx->slice_end = ~0ull;
    ctx->part = (uint32_t)ctx->rank;      // after cuts_set_dist: this rank's cyclic slice
    ctx->nparts = (uint32_t)ctx->world;   // of the shuffled level-1 list
    ctx->pre_j = 0;
    ctx->pre_count = 0;
    ctx->pre_rows = nullptr;
    ctx->has_query = true;
    return CUTS_OK;
}
}  // namespace

// ============================================================== C ABI
extern "C" {

int cuts_version(void) { return CUTS_ABI_VERSION; }

cuts_status cuts_create(cuts_ctx** out, const cuts_opts* o) {
    if (!out || !o) return CUTS_EINVAL;
    *out = nullptr;
    if (!o->arena || ((uintptr_t)o->arena % kAlign) != 0 || o->arena_bytes < (64u << 10)) return CUTS_EINVAL;
    cuts_ctx* ctx = new (std::nothrow) cuts_ctx();
    if (!ctx) return CUTS_ENOMEM;
    ctx->device = o->device;
    ctx->stream = (cudaStream_t)o->stream;
    ctx->arena = (char*)o->arena;
    ctx->arena_bytes = o->arena_bytes;
    ctx->seed = o->seed;
    ctx->ctrl = (unsigned long long*)ctx->arena;
    ctx->base_off = kCtrlBytes;
    cudaError_t e = cudaSetDevice(o->device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, o->device);
    if (e == cudaSuccess) e = cudaMallocHost((void**)&ctx->h_ctrl, 2 * kCtrlWords * sizeof(unsigned long long));
    if (e != cudaSuccess) {
        delete ctx;
        return CUTS_ECUDA;
    }
    *out = ctx;
    return CUTS_OK;
}

void cuts_destroy(cuts_ctx* ctx) {
    if (!ctx) return;
    if (ctx->comm && nccl().ok) nccl().destroy(ctx->comm);
    for (auto e : ctx->ev_pool) cudaEventDestroy(e);
    if (ctx->h_ctrl) cudaFreeHost(ctx->h_ctrl);
    delete ctx;
}

const char* cuts_last_error(const cuts_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

namespace {
cuts_status load_graph(cuts_ctx* ctx, uint32_t n, uint64_t nnz, const uint64_t* d_row_ptr,
                       const uint32_t* d_col, int validate, bool directed) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (!d_row_ptr || (nnz && !d_col)) return fail(ctx, CUTS_EINVAL, "null graph pointer");
    if (n == 0xFFFFFFFFu) return fail(ctx, CUTS_EINVAL, "n must be < 2^32-1");
    CK(cudaSetDevice(ctx->device));
    const uint64_t rows = directed ? 2ull * n : (uint64_t)n;   // directed: out-rows then in-rows
    if (rows >= 0xFFFFFFFFull) return fail(ctx, CUTS_EINVAL, "2n must be < 2^32-1 for a directed graph");
    uint64_t deg_bytes = align_up(rows * 4 + 4);
    if (kCtrlBytes + deg_bytes + (16u << 10) > ctx->arena_bytes) return fail(ctx, CUTS_ENOMEM, "arena too small for deg[%u]", n);
    ctx->has_graph = false;
    ctx->canon_valid = false;
    ctx->directed = directed;
    ctx->n = n;
    ctx->nnz = nnz;
    ctx->row_ptr = d_row_ptr;
    ctx->col = d_col;
    ctx->deg = (uint32_t*)(ctx->arena + kCtrlBytes);
    ctx->base_off = kCtrlBytes + deg_bytes;
    if (n) {
        unsigned grid = (unsigned)std::min<uint64_t>(((uint64_t)n + 255) / 256, (uint64_t)ctx->num_sms * 8);
        k_degree<<<grid, 256, 0, ctx->stream>>>(d_row_ptr, (uint32_t)rows, ctx->deg);
        CK(cudaGetLastError());
    }
    // row_ptr[0] == 0 and row_ptr[n] == nnz
    uint64_t ends[2] = {1, 0};
    CK(cudaMemcpyAsync(&ends[0], d_row_ptr, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(&ends[1], d_row_ptr + rows, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    if (ends[0] != 0 || ends[1] != nnz) return fail(ctx, CUTS_EINVAL, "row_ptr[0]=%llu row_ptr[n]=%llu nnz=%llu",
                                                    (unsigned long long)ends[0], (unsigned long long)ends[1], (unsigned long long)nnz);
    if (validate && n) {
        CK(cudaMemsetAsync(ctx->ctrl, 0, kCtrlWords * sizeof(unsigned long long), ctx->stream));
        Graph g{d_row_ptr, d_col, ctx->deg, nullptr, nullptr, n, 0, nullptr};
        g.dn = directed ? n : 0u;
        unsigned grid = (unsigned)std::min<uint64_t>((rows * 32 + 255) / 256, (uint64_t)ctx->num_sms * 16);
        k_validate<<<grid, 256, 0, ctx->stream>>>(g, ctx->ctrl);
        CK(cudaGetLastError());
        TRY(read_ctrl(ctx));
        if (ctx->h_ctrl[kErr]) return fail(ctx, CUTS_EINVAL, directed ?
            "digraph is not canonical (sorted, no loops/dups, ids < n, in-rows = transpose of out-rows)" :
            "graph is not canonical symmetric CSR (sorted, no loops/dups, ids < n)");
    }
    if (directed) {   // hub bitmaps and the packed stream assume one symmetric row per vertex
        ctx->nhubs = 0; ctx->hub_t_used = 0; ctx->hub = nullptr; ctx->bm = nullptr; ctx->colx = nullptr;
        ctx->has_graph = true;
        return CUTS_OK;
    }
    TRY(build_hubs(ctx));
    // packed candidate stream (degree filter without a gather) when ids fit 27 bits
    ctx->colx = nullptr;
    const uint64_t colx_bytes = align_up(nnz * 4);
    if (nnz && n <= kPackMask && ctx->base_off + colx_bytes + (ctx->arena_bytes / 2) <= ctx->arena_bytes &&
        !(ctx->debug & CUTS_DEBUG_NO_PACK)) {
        ctx->colx = (uint32_t*)(ctx->arena + ctx->base_off);
        unsigned grid = (unsigned)std::min<uint64_t>((nnz + 255) / 256, (uint64_t)ctx->num_sms * 16);
        k_pack<<<grid, 256, 0, ctx->stream>>>(d_col, nnz, ctx->deg, ctx->colx);
        CK(cudaGetLastError());
        ctx->base_off += colx_bytes;
    }
    ctx->has_graph = true;
    return CUTS_OK;
}
}  // namespace

cuts_status cuts_load_graph(cuts_ctx* ctx, uint32_t n, uint64_t nnz, const uint64_t* d_row_ptr,
                            const uint32_t* d_col, int validate) {
    return load_graph(ctx, n, nnz, d_row_ptr, d_col, validate, false);
}

cuts_status cuts_load_digraph(cuts_ctx* ctx, uint32_t n, uint64_t nnz, const uint64_t* d_row_ptr,
                              const uint32_t* d_col, int validate) {
    return load_graph(ctx, n, nnz, d_row_ptr, d_col, validate, true);
}

cuts_status cuts_set_hub_threshold(cuts_ctx* ctx, uint32_t t) {
    if (!ctx) return CUTS_EINVAL;
    ctx->hub_t = t;
    return CUTS_OK;
}

cuts_status cuts_set_query(cuts_ctx* ctx, uint32_t k, const uint32_t* row_ptr, const uint32_t* col,
                           const uint32_t* order) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (!ctx->has_graph) return fail(ctx, CUTS_ESTATE, "cuts_load_graph must precede cuts_set_query");
    QPlan qp{};
    ctx->has_query = false;
    TRY(plan_query(ctx, k, row_ptr, col, order, &qp));
    return finish_query(ctx, qp, false);
}

cuts_status cuts_set_query_directed(cuts_ctx* ctx, uint32_t k, const uint32_t* row_ptr, const uint32_t* col,
                                    const uint32_t* order) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (!ctx->has_graph) return fail(ctx, CUTS_ESTATE, "cuts_load_digraph must precede cuts_set_query_directed");
    QPlan qp{};
    ctx->has_query = false;
    TRY(plan_query_directed(ctx, k, row_ptr, col, order, &qp));
    return finish_query(ctx, qp, true);
}


cuts_status cuts_set_prefixes(cuts_ctx* ctx, uint32_t depth, uint64_t count, const uint32_t* d_prefixes) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (!ctx->has_query) return fail(ctx, CUTS_ESTATE, "cuts_set_query must precede cuts_set_prefixes");
    if (depth == 0) {                    // back to level-1 seeding
        ctx->pre_j = 0;
        ctx->pre_count = 0;
        ctx->pre_rows = nullptr;
        return CUTS_OK;
    }
    if (depth >= ctx->q.k) return fail(ctx, CUTS_EINVAL, "prefix depth %u must be < k = %u", depth, ctx->q.k);
    if (count && !d_prefixes) return fail(ctx, CUTS_EINVAL, "null prefix rows");
    if (count > kMaxLevel) return fail(ctx, CUTS_EINVAL, "too many prefixes (%llu)", (unsigned long long)count);
    ctx->pre_j = depth;
    ctx->pre_count = count;
    ctx->pre_rows = d_prefixes;
    return CUTS_OK;
}

cuts_status cuts_set_donation(cuts_ctx* ctx, cuts_poll_fn poll, cuts_ship_fn ship, void* user) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if ((poll == nullptr) != (ship == nullptr)) return fail(ctx, CUTS_EINVAL, "poll and ship must both be set or both NULL");
    ctx->poll = poll;
    ctx->ship = ship;
    ctx->user = user;
    return CUTS_OK;
}

cuts_status cuts_set_root_range(cuts_ctx* ctx, uint64_t begin, uint64_t end) {
    if (!ctx) return CUTS_EINVAL;
    if (!ctx->has_query) return fail(ctx, CUTS_ESTATE, "cuts_set_query must precede cuts_set_root_range");
    if (end < begin) return fail(ctx, CUTS_EINVAL, "root range end < begin");
    ctx->root_begin = begin;
    ctx->root_end = end;
    return CUTS_OK;
}

cuts_status cuts_set_root_slice(cuts_ctx* ctx, uint64_t begin, uint64_t end, uint32_t part, uint32_t nparts) {
    if (!ctx) return CUTS_EINVAL;
    if (!ctx->has_query) return fail(ctx, CUTS_ESTATE, "cuts_set_query must precede cuts_set_root_slice");
    if (end < begin || nparts == 0 || part >= nparts) return fail(ctx, CUTS_EINVAL, "bad root slice");
    ctx->slice_begin = begin;
    ctx->slice_end = end;
    ctx->part = part;
    ctx->nparts = nparts;
    return CUTS_OK;
}

cuts_status cuts_set_partition_depth(cuts_ctx* ctx, uint32_t depth) {
    if (!ctx) return CUTS_EINVAL;
    if (depth < 1 || depth >= (uint32_t)kMaxK) return fail(ctx, CUTS_EINVAL, "partition depth %u not in [1, %d)", depth, kMaxK);
    ctx->part_depth = depth;
    return CUTS_OK;
}

cuts_status cuts_partition_size(cuts_ctx* ctx, uint64_t* n) {
    if (!ctx || !n) return CUTS_EINVAL;
    if (!ctx->has_graph || !ctx->has_query) return fail(ctx, CUTS_ESTATE, "load_graph and set_query must precede cuts_partition_size");
    const int k = (int)ctx->q.k;
    if (ctx->part_depth <= 1 || (int)ctx->part_depth >= k) {
        uint64_t nc = 0;
        return cuts_level1_size(ctx, &nc, n);
    }
    ctx->size_only = true;
    const cuts_status s = run_query(ctx, CUTS_HYBRID, false, nullptr, 0);
    ctx->size_only = false;
    TRY(s);
    *n = ctx->st.level_size[ctx->part_depth];
    return CUTS_OK;
}

cuts_status cuts_level1_size(cuts_ctx* ctx, uint64_t* canonical, uint64_t* in_range) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (!ctx->has_graph || !ctx->has_query) return fail(ctx, CUTS_ESTATE, "load_graph and set_query must precede cuts_level1_size");
    CK(cudaSetDevice(ctx->device));
    TRY(ensure_canonical(ctx));
    const uint64_t nc = ctx->canon_n;
    const uint64_t rb = std::min(ctx->root_begin, nc), re = std::max(rb, std::min(ctx->root_end, nc));
    if (canonical) *canonical = nc;
    if (in_range) *in_range = re - rb;
    return CUTS_OK;
}

cuts_status cuts_count(cuts_ctx* ctx, cuts_mode mode, uint64_t* out) {
    if (!ctx || !out) return CUTS_EINVAL;
    ctx->err.clear();
    TRY(run_query(ctx, mode, false, nullptr, 0));
    *out = ctx->st.count_lo;
    if (ctx->st.count_hi) return fail(ctx, CUTS_EOVERFLOW, "count >= 2^64 (hi word %llu)", (unsigned long long)ctx->st.count_hi);
    return CUTS_OK;
}

cuts_status cuts_enumerate(cuts_ctx* ctx, cuts_mode mode, uint32_t* d_out, uint64_t cap_rows, uint64_t* n_found) {
    if (!ctx || !n_found) return CUTS_EINVAL;
    ctx->err.clear();
    TRY(run_query(ctx, mode, true, d_out, cap_rows));
    *n_found = ctx->st.count_lo;
    if (*n_found > cap_rows) return fail(ctx, CUTS_ETRUNC, "found %llu rows, cap %llu", (unsigned long long)*n_found, (unsigned long long)cap_rows);
    return CUTS_OK;
}

cuts_status cuts_get_stats(const cuts_ctx* ctx, cuts_stats* out) {
    if (!ctx || !out) return CUTS_EINVAL;
    *out = ctx->st;
    return CUTS_OK;
}

cuts_status cuts_set_debug(cuts_ctx* ctx, uint32_t flags) {
    if (!ctx) return CUTS_EINVAL;
    ctx->debug = flags;
    return CUTS_OK;
}

cuts_status cuts_debug_group_hist(cuts_ctx* ctx, uint64_t* out) {
    if (!ctx || !out) return CUTS_EINVAL;
    CK(cudaSetDevice(ctx->device));
    CK(cudaMemcpyAsync(out, ctx->ctrl + kGroupHist, kGroupHistWords * sizeof(unsigned long long),
                       cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return CUTS_OK;
}

cuts_status cuts_trie_decode(cuts_ctx* ctx, uint32_t nlevels, const uint64_t* sizes, const uint32_t* const* d_ca,
                             const uint32_t* const* d_pa, uint32_t* d_out) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (nlevels == 0 || nlevels > CUTS_MAX_K || !sizes || !d_ca || !d_pa) return fail(ctx, CUTS_EINVAL, "bad trie arguments");
    CK(cudaSetDevice(ctx->device));
    DecodeArgs a{};
    a.L = nlevels;
    for (uint32_t l = 0; l < nlevels; ++l) {
        a.ca[l] = d_ca[l];
        a.pa[l] = l ? d_pa[l] : nullptr;
        a.size[l] = sizes[l];
        if (!a.ca[l] || (l && sizes[l] && !a.pa[l])) return fail(ctx, CUTS_EINVAL, "null level %u", l);
    }
    CK(cudaMemsetAsync(ctx->ctrl, 0, kCtrlWords * sizeof(unsigned long long), ctx->stream));
    uint64_t n = sizes[nlevels - 1];
    if (n) {
        unsigned grid = (unsigned)std::min<uint64_t>((n + 255) / 256, (uint64_t)ctx->num_sms * 8);
        k_trie_decode<<<grid, 256, 0, ctx->stream>>>(a, d_out, ctx->ctrl);
        CK(cudaGetLastError());
    }
    TRY(read_ctrl(ctx));
    if (ctx->h_ctrl[kErr]) return fail(ctx, CUTS_EINVAL, "parent index out of range");
    return CUTS_OK;
}

cuts_status cuts_dist_unique_id(void* out_128B) {
    if (!out_128B) return CUTS_EINVAL;
    NcclApi& api = nccl();
    if (!api.ok) return CUTS_ECOMM;
    ncclUniqueId id;
    if (api.get_unique_id(&id) != ncclSuccess) return CUTS_ECOMM;
    static_assert(sizeof(ncclUniqueId) == CUTS_DIST_UID_BYTES, "ncclUniqueId size");
    memcpy(out_128B, &id, sizeof id);
    return CUTS_OK;
}

cuts_status cuts_set_dist(cuts_ctx* ctx, int rank, int world, const void* nccl_uid_128B, const void* peers) {
    if (!ctx) return CUTS_EINVAL;
    ctx->err.clear();
    if (world < 1 || rank < 0 || rank >= world) return fail(ctx, CUTS_EINVAL, "bad rank %d / world %d", rank, world);
    if (peers) return fail(ctx, CUTS_EINVAL, "peers is reserved and must be NULL");
    if (world > 1 && !nccl_uid_128B) return fail(ctx, CUTS_EINVAL, "world %d needs an NCCL unique id", world);
    CK(cudaSetDevice(ctx->device));
    NcclApi& api = nccl();
    if (ctx->comm) {
        if (api.ok) api.destroy(ctx->comm);
        ctx->comm = nullptr;
    }
    if (nccl_uid_128B) {   // world 1 with an id still builds a (trivial) communicator
        if (!api.ok) return fail(ctx, CUTS_ECOMM, "libnccl.so.2 not found (dlopen)");
        ncclUniqueId id;
        memcpy(&id, nccl_uid_128B, sizeof id);
        const ncclResult_t r = api.init_rank(&ctx->comm, world, id, rank);
        if (r != ncclSuccess) {
            ctx->comm = nullptr;
            return fail(ctx, CUTS_ECOMM, "ncclCommInitRank(world %d, rank %d): %s", world, rank, api.error_string(r));
        }
    }
    ctx->rank = rank;
    ctx->world = world;
    ctx->part = (uint32_t)rank;
    ctx->nparts = (uint32_t)world;
    return CUTS_OK;
}

cuts_status cuts_allreduce_count(cuts_ctx* ctx, uint64_t lo, uint64_t hi, uint64_t* out_lo, uint64_t* out_hi) {
    if (!ctx || !out_lo || !out_hi) return CUTS_EINVAL;
    ctx->err.clear();
    if (ctx->world == 1 && !ctx->comm) {
        *out_lo = lo;
        *out_hi = hi;
        return CUTS_OK;
    }
    if (!ctx->comm) return fail(ctx, CUTS_ESTATE, "cuts_set_dist with an NCCL id must precede cuts_allreduce_count");
    CK(cudaSetDevice(ctx->device));
    // four 32-bit limbs in u64 words: each limb sum is <= world * (2^32 - 1), no overflow
    unsigned long long* h = ctx->h_ctrl + kCtrlWords + 8;
    unsigned long long* d = ctx->ctrl + kDistLimbs;
    h[0] = lo & 0xffffffffull; h[1] = lo >> 32; h[2] = hi & 0xffffffffull; h[3] = hi >> 32;
    CK(cudaMemcpyAsync(d, h, 4 * sizeof(unsigned long long), cudaMemcpyHostToDevice, ctx->stream));
    const ncclResult_t r = nccl().all_reduce(d, d, 4, ncclUint64, ncclSum, ctx->comm, ctx->stream);
    if (r != ncclSuccess) return fail(ctx, CUTS_ECOMM, "ncclAllReduce: %s", nccl().error_string(r));
    CK(cudaMemcpyAsync(h, d, 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    unsigned __int128 t = (unsigned __int128)h[0] + ((unsigned __int128)h[1] << 32) + ((unsigned __int128)h[2] << 64) +
                          ((unsigned __int128)h[3] << 96);
    *out_lo = (uint64_t)t;
    *out_hi = (uint64_t)(t >> 64);
    return CUTS_OK;
}

}  // extern "C"
