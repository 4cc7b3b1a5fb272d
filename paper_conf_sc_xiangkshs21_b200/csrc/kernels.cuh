// kernels.cuh — sm_100a device code for the cuTS hot path.
// "P:n" cites /root/reference/PAPER.md line n; design in DESIGN.md §4.
//
// Pipeline per level j -> j+1 (one window of W entries of the level-j trie):
//   k_plan<J>      : per entry, walk the trie path (J-1 parent hops),
//                    pick the smallest backward-neighbour list as the candidate
//                    source (c-intersection initial set, Alg. 2 l.22-23), emit
//                    ub(e) = its length (a never-exceeded bound on children).
//   exclusive scan : offs = prefix(ub)  ->  flat candidate-item space.
//   k_extend<J,M>  : load-balanced over items (each thread one (entry, candidate)
//                    pair, so hub lists are split across CTAs): membership of the
//                    candidate in every other backward list (binary search in the
//                    sorted CSR row), degree filter (Def. 5),
//                    injectivity, then warp-aggregated output slots
//                    (ballot/popc + one atomic per warp) and the write
//                    of (vertex, parent) into level j+1 — or a count (last level),
//                    or a full row in query-id order (enumerate).
#pragma once
#include <cstdint>

namespace cuts {

constexpr int kMaxK = 8;
constexpr int kLrMaxM = 512;                // local rows: largest sibling group held in shared memory
constexpr int kLrWords = kLrMaxM / 32;
constexpr int kLrBatch = 256;              // k_lr_group: parent slots claimed per CTA fetch
constexpr int kDlrMaxM = 1024;             // deep local rows: largest sibling group (16 u64 words per row)
constexpr uint32_t kDlrSmemBytes = 32u << 10;   // k_dlr_tail_cta: row blocks staged in shared memory up to this
constexpr int kTile = 256;   // items per CTA tile == threads per CTA

struct QPlan {                 // query in matching-order positions
    uint32_t k;
    uint32_t S[kMaxK];         // S[i] = query vertex matched at position i
    uint32_t qdeg[kMaxK];      // deg_Q(S[i])       (degree filter)
    uint32_t bw[kMaxK];        // bit p set <=> (S[p], S[i]) in E_Q, p < i (next_neigh)
    // bw[i] == 0, i > 0: S[i] starts another connected component of Q.
    // Its candidates are the cross product's factor {v : deg(v) >= qdeg[i]}, a
    // sorted list at Graph::fre + foff[i] of flen[i] entries (built per run).
    uint64_t foff[kMaxK];
    uint32_t flen[kMaxK];
    // directed Q (NEXT-1): bw[i] bit p <=> arc S[p] -> S[i] (candidate
    // in children(f(S[p])), c-intersection); bwi[i] bit p <=> arc S[i] -> S[p]
    // (candidate in parents(f(S[p])), p-intersection, Alg. 2 l.33-42).  qdeg is
    // then the out-degree and qdin the in-degree (Def. 5 with P:262-264).
    uint32_t bwi[kMaxK];
    uint32_t qdin[kMaxK];
    uint32_t src_first;        // ablation: source = first backward list (Alg. 2 a1), not the shortest
    uint32_t count_fast;       // cuts_count: set-difference count at a single-list last level
};

// Count-only last level with ONE backward list and no degree bound:
// the children of an entry are list \ path, so their number is |list| minus the
// path vertices found in the list (<= J binary searches) — the exact size of the
// intersection result without streaming the list.
template <int J>
__device__ __forceinline__ bool fast_last(const QPlan& q, uint32_t need, uint32_t qmin) {
    return q.count_fast && J + 1 == (int)q.k && __popc(need) == 1 && q.qdeg[J] <= qmin && q.qdin[J] == 0;
}

struct Trie {                  // lv[l] = level l (1-based): .x = data vertex, .y = parent index in level l-1
    const uint2* lv[kMaxK];
};

// Ancestor-set reuse ("incremental intersection").  Level a+1 was
// written ORDERED: the children of level-a entry x are the contiguous range
// [cpos[x-w0] - cpos[ea], cpos[x-w0+1] - cpos[ea]) of the level-(a+1) chunk
// lv, and their vertices are exactly {c in the intersection of N(f(S[p])),
// p in bw[a] : deg(c) >= qdeg[a], c not on x's path}.  When bw[a] is a subset
// of bw[J] and qdeg[a] <= qdeg[J], that range contains every candidate of a
// level-J descendant of x, so it can replace the lists of bw[a] as the source.
struct Reuse {
    const uint2* lv;           // level a+1 chunk (candidate source for trie-sourced entries)
    const uint64_t* cpos;      // level a window's exclusive scan of child counts
    uint64_t w0;               // level a window start
    uint64_t ea;               // first level-a entry (window-relative) of the level a+1 chunk
    uint32_t a;                // ancestor level (0: off)
    uint32_t bwa;              // bw[a]
    // symmetric last level ("pair sharing"): a = J-1 and the only list left
    // to test is the entry's own N(f(S[J-1])), so sibling c_j is a child of sibling c_i iff
    // {c_i, c_j} is an edge — the relation is symmetric.  Each entry then streams only the
    // siblings AFTER itself and the count-only kernel doubles its sum (every unordered
    // sibling pair tested once instead of twice)
    uint32_t sym;
    // local rows took this level's sibling groups of <= skip_small members (0: none):
    // k_plan gives their entries no candidates (ub = 0) so the windowed pipeline only
    // sees the rest
    uint32_t skip_small;
};

constexpr uint64_t kTrieSrc = 1ull << 63;   // src_off flag: the source is a trie range
constexpr uint64_t kFreeSrc = 1ull << 62;   // src_off flag: the source is a component's free list
constexpr uint64_t kIdSrc = 1ull << 61;     // with kFreeSrc: the identity list [0, n) (degree filter in-kernel)
constexpr uint32_t kSkip = 0xffffffffu;     // list-slot length: no list in this slot

struct Graph {
    const uint64_t* __restrict__ row_ptr;
    const uint32_t* __restrict__ col;
    const uint32_t* __restrict__ deg;
    const uint32_t* __restrict__ hub;   // hub[v] = row of v in bm, or kNoHub (nullptr: no bitmaps)
    const uint32_t* __restrict__ bm;    // hub adjacency bitmaps, words u32 per row
    uint32_t n;
    uint32_t words;
    const uint32_t* __restrict__ colx;  // col with min(deg, 31) packed in bits 27..31 (nullptr: n >= 2^27)
    const uint32_t* __restrict__ fre = nullptr;   // free lists of component roots (QPlan::foff/flen)
    uint32_t dn = 0;   // directed: rows [0,n) are out-lists, rows [n,2n) in-lists, dn = n; undirected: 0
    // hub-to-hub core bitmap: row h (a hub) has bit hub[u] set for every hub neighbour u —
    // nhubs^2 bits (32 MB at 16 K hubs), small enough to stay in L2 (nullptr: none)
    const uint32_t* __restrict__ cb = nullptr;
    uint32_t cbw = 0;  // u32 words per core row
};

// is c in N(v) for a hub v with bitmap row h: the L2-resident core row when c is a hub
// too, else the full n-bit row
__device__ __forceinline__ bool hub_probe(const Graph& g, uint32_t h, uint32_t c) {
    if (g.cb) {
        const uint32_t hc = __ldg(g.hub + c);
        if (hc != 0xffffffffu) return (__ldg(g.cb + (uint64_t)h * g.cbw + (hc >> 5)) >> (hc & 31)) & 1u;
    }
    return (__ldg(g.bm + (uint64_t)h * g.words + (c >> 5)) >> (c & 31)) & 1u;
}

constexpr uint32_t kNoHub = 0xffffffffu;
constexpr int kPackShift = 27;               // colx: vertex id in bits 0..26, min(deg, 31) above
constexpr uint32_t kPackMask = (1u << kPackShift) - 1u;
constexpr uint32_t kBmFlag = 0x80000000u;   // list-slot length flag: probe a bitmap instead

enum Mode { kWrite = 0, kCount = 1, kEnum = 2 };

// control block (u64 words in the arena)
// algorithmic bytes (CUTS_DEBUG_BYTES; SURVEY §8.d model, frozen): kBytesPlan = entry + path
// hops + list bounds; kBytesExt = every backward list read once (4 d per list, whatever
// source the kernel streams) + 4 per intersection survivor; kBytesOut = children written;
// kBytesNeed = the source bytes this kernel's algorithm actually needs (shortest list,
// ancestor range, or the set-difference searches), reported beside the model
enum Ctrl { kCursor = 0, kCountLo = 1, kCountHi = 2, kErr = 3, kBytesPlan = 4, kBytesExt = 5,
            kEnumCursor = 6, kNumSel = 7, kWork = 8, kBytesOut = 9, kBytesNeed = 10, kFind = 24,
            kBins = 12, kLrLevel = 15, kLrLarge = 29, kLrWork = 30, kDlrLarge = 31, kDlrWork = 32, kTailOps = 33, kDistLimbs = 56, kCtrlWords = 64,
            kGroupHist = 64, kGroupHistWords = 432 };   // CUTS_DEBUG_GROUPS: [level][16 buckets][3]

__device__ __forceinline__ void add_u128(unsigned long long* lo_hi, unsigned long long v) {
    if (v == 0) return;
    unsigned long long old = atomicAdd(lo_hi, v);
    if (old + v < old) atomicAdd(lo_hi + 1, 1ull);
}

__device__ __forceinline__ unsigned long long warp_sum(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// first position in sorted col[b, e) holding value c, or false
__device__ __forceinline__ bool list_contains(const uint32_t* __restrict__ col, uint64_t b, uint64_t e,
                                              uint32_t c) {
    // branch-light lower bound
    uint64_t len = e - b;
    const uint32_t* base = col + b;
    while (len > 1) {
        uint64_t half = len >> 1;
        if (__ldg(base + half - 1) < c) base += half;   // move past the lower half
        len -= half;
    }
    return len == 1 && __ldg(base) == c;
}

// ------------------------------------------------------------------ degrees
__global__ void k_degree(const uint64_t* __restrict__ row_ptr, uint32_t n, uint32_t* __restrict__ deg) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x)
        deg[v] = (uint32_t)(row_ptr[v + 1] - row_ptr[v]);
}

// colx[p] = col[p] | min(deg(col[p]), 31) << 27: the candidate stream carries the
// degree-filter input (Def. 5), so the filter costs no random 4 B gather
__global__ void k_pack(const uint32_t* __restrict__ col, uint64_t nnz, const uint32_t* __restrict__ deg,
                       uint32_t* __restrict__ colx) {
    for (uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; p < nnz; p += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t u = col[p];
        colx[p] = u | (min(deg[u], 31u) << kPackShift);
    }
}

// SV-style membership rows (Alg. 2 l.7-17's |V|-sized scatter vector, P:1055-1072,
// precomputed once per hub vertex instead of per worker): for every vertex with
// deg >= T a bitmap over [0, n); a membership test against a hub list is then
// one load instead of a binary search.
__global__ void k_hub_hist(const uint32_t* __restrict__ deg, uint32_t n, unsigned long long* __restrict__ hist) {
    // hist[b] = #vertices with deg >= 2^b, b < 32
    __shared__ unsigned int s[32];
    if (threadIdx.x < 32) s[threadIdx.x] = 0;
    __syncthreads();
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const uint32_t d = deg[v];
        if (d) atomicAdd(&s[31 - __clz(d)], 1u);
    }
    __syncthreads();
    if (threadIdx.x < 32 && s[threadIdx.x]) atomicAdd(hist + threadIdx.x, (unsigned long long)s[threadIdx.x]);
}

__global__ void k_hub_mark(const uint32_t* __restrict__ deg, uint32_t n, uint32_t t, uint32_t* __restrict__ hub,
                           unsigned long long* __restrict__ counter) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x)
        hub[v] = deg[v] >= t ? (uint32_t)atomicAdd(counter, 1ull) : kNoHub;
}

// one warp per vertex: hubs set the bits of their neighbours
__global__ void k_hub_fill(const uint64_t* __restrict__ row_ptr, const uint32_t* __restrict__ col, uint32_t n,
                           const uint32_t* __restrict__ hub, uint32_t words, uint32_t* __restrict__ bm,
                           uint32_t* __restrict__ cb, uint32_t cbw) {
    const int lane = threadIdx.x & 31;
    const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t v = warp; v < n; v += nwarps) {
        const uint32_t h = hub[v];
        if (h == kNoHub) continue;
        uint32_t* row = bm + (uint64_t)h * words;
        for (uint64_t p = row_ptr[v] + lane; p < row_ptr[v + 1]; p += 32) {
            const uint32_t u = col[p];
            atomicOr(row + (u >> 5), 1u << (u & 31));
            if (cb) {
                const uint32_t hu = hub[u];
                if (hu != kNoHub) atomicOr(cb + (uint64_t)h * cbw + (hu >> 5), 1u << (hu & 31));
            }
        }
    }
}

// graph validation: sorted strictly ascending rows, no loops, ids < n, symmetric
// (directed: the in-rows are the transpose of the out-rows).
// one warp per row; sets ctrl[kErr] = 1 on any violation.
__global__ void k_validate(Graph g, unsigned long long* ctrl) {
    const int lane = threadIdx.x & 31;
    const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t r = warp; r < (uint64_t)g.n + g.dn; r += nwarps) {
        const uint64_t v = r < g.n ? r : r - g.n;
        uint64_t b = g.row_ptr[r], e = g.row_ptr[r + 1];
        bool bad = e < b;
        for (uint64_t p = b + lane; !bad && p < e; p += 32) {
            uint32_t u = g.col[p];
            if (u >= g.n || u == v) { bad = true; break; }
            if (p > b && g.col[p - 1] >= u) { bad = true; break; }
            const uint64_t o = r < g.n ? (uint64_t)u + g.dn : (uint64_t)u;   // the opposite row of u
            if (!list_contains(g.col, g.row_ptr[o], g.row_ptr[o + 1], (uint32_t)v)) { bad = true; break; }
        }
        if (__any_sync(0xffffffffu, bad) && lane == 0) atomicExch(ctrl + kErr, 1ull);
    }
}

// ---------------------------------------------------------------- level 1
// canonical level-1 flags: deg(v) >= deg_Q(S[0])  (Alg. 1 l.8-11)
struct DegAtLeast {   // directed: deg[v] = out-degree, deg[dn + v] = in-degree
    const uint32_t* deg; uint32_t t; uint32_t dn = 0; uint32_t ti = 0;
    __host__ __device__ bool operator()(uint32_t v) const { return deg[v] >= t && (ti == 0 || deg[dn + v] >= ti); }
};

// seeded bijection on [0, R) (4-round Feistel + cycle walking): the randomised
// partial-path placement of P:916-922 (reading P25: level 1 only, performance only)
struct Shuffle {
    uint64_t R; uint32_t half; uint32_t mask; uint64_t key[4];
    __device__ __forceinline__ static uint32_t mix(uint64_t x) {
        x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
        return (uint32_t)x;
    }
    __device__ __forceinline__ uint64_t apply(uint64_t p) const {
        do {
            uint32_t l = (uint32_t)(p >> half) & mask, r = (uint32_t)p & mask;
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                uint32_t nl = r;
                r = l ^ (mix(key[i] ^ r) & mask);
                l = nl;
            }
            p = ((uint64_t)l << half) | r;
        } while (p >= R);
        return p;
    }
};

// L1[i] = canon[rb + pi(p0 + i*nparts)], i < cnt
__global__ void k_level1(const uint32_t* __restrict__ canon, uint64_t rb, Shuffle sh, uint64_t p0,
                         uint32_t nparts, uint64_t cnt, uint2* __restrict__ L1) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t p = p0 + i * nparts;
        L1[i] = make_uint2(canon[rb + sh.apply(p)], 0u);
    }
}

// enumerate rows for k == 1
__global__ void k_rows_k1(const uint2* __restrict__ L1, uint64_t cnt, uint32_t* __restrict__ rows,
                          uint64_t cap) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt && i < cap;
         i += (uint64_t)gridDim.x * blockDim.x)
        rows[i] = L1[i].x;
}

// ---------------------------------------------------------------- plan
// J = number of matched positions of the entries (= next position to match).
// One thread per entry: walk the trie path, read the bounds of the
// backward-neighbour lists bw[J], take the shortest as the candidate source
// (c-intersection initial set, Alg. 2 l.22-23) and emit ub(e) = its length, a
// never-exceeded bound on the entry's children.  The other lists are written
// as descriptors sorted by length (shortest first; hub lists as bitmap rows,
// which sort last), so the extend kernel's virtual warps read them instead of
// recomputing them lane-redundantly.
//   lst_off[x*W + e]: element offset into col (or into bm for a bitmap row)
//   lst_len[x*W + e]: list length, | kBmFlag for a bitmap row
template <int J, bool D>
__global__ void __launch_bounds__(256) k_plan(Graph g, Trie t, QPlan q, uint64_t w0, uint32_t W,
                                              uint32_t* __restrict__ path_s,
                                              uint64_t* __restrict__ src_off,
                                              uint64_t* __restrict__ ub,
                                              uint64_t* __restrict__ lst_off,
                                              uint32_t* __restrict__ lst_len,
                                              unsigned long long* __restrict__ ctrl, int count_bytes, Reuse ru) {
    const uint32_t bw = q.bw[J];
    const uint32_t bwi = q.bwi[J];
    constexpr int J2 = D ? 2 * J : J;   // list slots: [0, J) children of path[p], [J, 2J) parents (directed)
    unsigned long long bytes_plan = 0, bytes_ext = 0, bytes_need = 0;
    for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e <= W; e += gridDim.x * blockDim.x) {
        if (e == W) { ub[W] = 0; continue; }
        uint32_t path[J];
        uint2 cur = t.lv[J][w0 + e];
        path[J - 1] = cur.x;
        uint32_t idx = cur.y;
        if (!D && ru.sym && !count_bytes) {
            // symmetric last level: the parent IS the ancestor (a = J-1) and the only list
            // left is the entry's own; siblings never hold a path vertex, so no trie walk
            const uint64_t k0 = (uint64_t)idx - ru.w0;
            const uint64_t me = w0 + e + 1;
            src_off[e] = me | kTrieSrc;
            ub[e] = ru.cpos[k0 + 1] - ru.cpos[ru.ea] - me;
            const uint32_t v = cur.x;
            const uint32_t h = g.hub ? __ldg(g.hub + v) : kNoHub;
            uint64_t off;
            uint32_t len;
            if (h != kNoHub) { off = (uint64_t)h * g.words; len = kBmFlag; }
            else { off = g.row_ptr[v]; len = (uint32_t)(g.row_ptr[v + 1] - off); }
            lst_off[e] = off;      // slot 0 only: the extend launch for this level has NL = 1
            lst_len[e] = len;
            path_s[(size_t)(J - 1) * W + e] = v;   // and reads path[J-1] only (pmin = J-1)
            continue;
        }
        if (ru.skip_small) {
            const uint64_t k0 = (uint64_t)idx - ru.w0;   // the parent is the ancestor (a = J-1)
            if (ru.cpos[k0 + 1] - ru.cpos[k0] <= (uint64_t)ru.skip_small) {
                ub[e] = 0;
                src_off[e] = 0;
                continue;
            }
        }
        uint32_t xa = 0;                             // index of the level-a ancestor (reuse)
#pragma unroll
        for (int p = J - 2; p >= 0; --p) {          // trie walk
            if (p + 1 == (int)ru.a) xa = idx;
            cur = t.lv[p + 1][idx];
            path[p] = cur.x;
            idx = cur.y;
        }
        uint64_t lb_[J2];
        uint32_t ln_[J2];
        uint64_t lists = 0, best_b = 0;
        uint32_t best_d = 0xffffffffu;
        int best = -1;
        const uint32_t need = D ? (bw | (bwi << J)) : bw;
#pragma unroll
        for (int s = 0; s < J2; ++s) {
            ln_[s] = 0xffffffffu;
            lb_[s] = 0;
            if ((need >> s) & 1u) {
                const uint64_t row = s < J ? (uint64_t)path[s] : (uint64_t)path[s - J] + g.dn;
                const uint64_t b = g.row_ptr[row];
                const uint32_t d = (uint32_t)(g.row_ptr[row + 1] - b);
                lists += d;
                lb_[s] = b;
                ln_[s] = d;
                if (best < 0 || (!q.src_first && d < best_d)) { best = s; best_d = d; best_b = b; }
            }
        }
        // ancestor-set source: the children range of the level-a ancestor replaces
        // the lists of bw[a] when it is no longer than every remaining list
        uint32_t keep = need;                        // lists still to be tested
        bool trie = false;
        uint64_t trie_off = 0, rest_sum = 0;
        uint32_t trie_len = 0;
        if (ru.a) {
            const uint64_t k0 = (uint64_t)xa - ru.w0;
            const uint64_t c0 = ru.cpos[k0], base = ru.cpos[ru.ea];
            trie_len = (uint32_t)(ru.cpos[k0 + 1] - c0);
            trie_off = c0 - base;
            uint32_t rest_min = 0xffffffffu;
#pragma unroll
            for (int p = 0; p < J; ++p)
                if (((bw & ~ru.bwa) >> p) & 1u) { rest_min = min(rest_min, ln_[p]); rest_sum += ln_[p]; }
            if (ru.sym) {        // the siblings after this entry (w0 + e is its index in the chunk)
                const uint64_t me = w0 + e + 1;
                trie_len = (uint32_t)(ru.cpos[k0 + 1] - base - me);
                trie_off = me;
                trie = true;
                keep = bw & ~ru.bwa;
            } else if (trie_len <= rest_min) { trie = true; keep = bw & ~ru.bwa; }
        }
        if (need == 0) {         // component root: cross-product factor
            src_off[e] = q.foff[J] | kFreeSrc;
            ub[e] = q.flen[J];
            lists = q.flen[J];
        } else if (trie) {
            src_off[e] = trie_off | kTrieSrc;
            ub[e] = trie_len;
            best = -1;
        } else {
            src_off[e] = best_b;
            ub[e] = best_d;
        }
        // other lists: hub rows become bitmap probes; then sort by length
        int x = 0;
#pragma unroll
        for (int p = 0; p < J2; ++p) {
            if (p != best && ((keep >> p) & 1u)) {
                // hub bitmaps cover out-rows of an undirected graph only (g.hub is null when directed)
                const uint32_t h = (g.hub && p < J) ? __ldg(g.hub + path[p]) : kNoHub;
                if (h != kNoHub) { lb_[p] = (uint64_t)h * g.words; ln_[p] |= kBmFlag; }
            } else {
                ln_[p] = 0xffffffffu;     // not a list to test (the source, or not backward)
            }
        }
#pragma unroll
        for (int i = 0; i < J2; ++i)
#pragma unroll
            for (int y = 0; y + 1 < J2 - i; ++y)
                if (ln_[y + 1] < ln_[y]) {
                    const uint32_t tl = ln_[y]; ln_[y] = ln_[y + 1]; ln_[y + 1] = tl;
                    const uint64_t tb = lb_[y]; lb_[y] = lb_[y + 1]; lb_[y + 1] = tb;
                }
        const int nl = __popc(need) - 1;   // -1 for a component root: no lists (host: nl <= J-1)
#pragma unroll
        for (int y = 0; y < J - 1; ++y)
            if (y < nl) {
                lst_off[(size_t)y * W + e] = lb_[y];
                lst_len[(size_t)y * W + e] = ln_[y];
            }
        (void)x;
#pragma unroll
        for (int p = 0; p < J; ++p) path_s[(size_t)p * W + e] = path[p];
        if (count_bytes) {   // 8 (entry) + 8(J-1) (hops) + 16 per list bound
            bytes_plan += 8ull + 8ull * (J - 1) + 16ull * __popc(need);
            bytes_ext += 4ull * lists;                   // the model: every backward list read once
            if (trie) {          // needed: the ancestor range (8 B entries) + the lists not covered by it
                bytes_need += 8ull * trie_len + 4ull * rest_sum;
            } else if (fast_last<J>(q, need, g.dn ? 0u : 1u)) {   // J binary searches in the list
                bytes_need += 4ull * J * (32 - __clz(best_d));
            } else {
                bytes_need += 4ull * lists;
            }
        }
    }
    if (count_bytes) {
        bytes_plan = warp_sum(bytes_plan);
        bytes_ext = warp_sum(bytes_ext);
        bytes_need = warp_sum(bytes_need);
        if ((threadIdx.x & 31) == 0) {
            atomicAdd(ctrl + kBytesPlan, bytes_plan);
            atomicAdd(ctrl + kBytesExt, bytes_ext);
            atomicAdd(ctrl + kBytesNeed, bytes_need);
        }
    }
}

// ---------------------------------------------------------------- extend
// Items [t0, t1) of the window's flat candidate space (offs = exclusive scan of
// ub, W+1 entries, ub(e) = |source list|).  J = matched positions of the
// parents; the child takes position J.  NL = |bw[J]| - 1 lists to test besides
// the source (a compile-time constant per level).
//
// Mapping: a virtual warp of G lanes per entry (the paper's single-bin virtual
// warps sized from the average degree), entries fetched dynamically
// in batches.  The G lanes walk the source list G candidates at a time
// (coalesced), apply injectivity and the degree filter (Def. 5),
// probe the hub lists' bitmaps (loads issued together), then test membership
// in the remaining sorted lists, shortest first, each by a branch-free binary
// search from a per-list cursor that only moves forward (candidates arrive in
// ascending order).  Output: one ballot and one atomic per warp per chunk
// (P:704-708).
//
// M: kWrite -> level J+1 entries (vertex, parent = w0 + e) at ctrl[kCursor]
// (dropped past cap; HYBRID sizes cap so that never happens); kCount -> 128-bit
// count; kEnum -> rows of k u32 in query-id order at ctrl[kEnumCursor].
template <int J, int NL, int M, int G>
__global__ void __launch_bounds__(256, (NL == 0 || (J <= 3 && NL < 2)) ? 6 : (J <= 5 ? 5 : 4)) k_extend(Graph g, QPlan q, uint64_t w0, uint32_t W,
                                               const uint32_t* __restrict__ path_s,
                                               const uint64_t* __restrict__ src_off,
                                               const uint64_t* __restrict__ offs,
                                               const uint64_t* __restrict__ lst_off,
                                               const uint32_t* __restrict__ lst_len,
                                               uint64_t t0, uint64_t t1,
                                               uint2* __restrict__ out_level,
                                               uint32_t* __restrict__ out_rows, uint64_t cap,
                                               unsigned long long* __restrict__ ctrl, int count_bytes,
                                               uint32_t batch, uint32_t qda, const uint2* __restrict__ rsrc,
                                               uint64_t* __restrict__ ord_cnt,
                                               const uint64_t* __restrict__ ord_pos, uint32_t ord_ea,
                                               const uint32_t* __restrict__ elist, uint32_t elist_n,
                                               uint32_t cmul, uint32_t pmin) {
    constexpr int VPW = 32 / G;
    constexpr unsigned kGMask = G == 32 ? 0xffffffffu : ((1u << G) - 1u);
    constexpr int NLA = NL > 0 ? NL : 1;
    __shared__ uint32_t s_ent[2];
    if (threadIdx.x == 0 && !elist) {        // entries holding items t0 and t1-1
        uint64_t tt[2] = {t0, t1 - 1};
        for (int z = 0; z < 2; ++z) {
            uint32_t lo = 0, hi = W - 1;
            while (lo < hi) {
                uint32_t mid = (lo + hi + 1) >> 1;
                if (offs[mid] <= tt[z]) lo = mid; else hi = mid - 1;
            }
            s_ent[z] = lo;
        }
    }
    __syncthreads();
    // binned launch (CUTS_DEBUG_BINNED): the entries are an explicit list (one bin)
    const uint32_t ea = elist ? 0u : s_ent[0];
    const uint32_t nent = elist ? elist_n : s_ent[1] - ea + 1;
    const int lane = threadIdx.x & 31;
    const int vl = lane & (G - 1);
    const int vb = lane & ~(G - 1);
    const uint32_t qd = q.qdeg[J];
    const uint32_t qdi = q.qdin[J];              // directed: in-degree bound (0: none)
    // undirected: a candidate from a list has deg >= 1, so qdeg <= 1 needs no check;
    // directed: a child may have out-degree 0
    const uint32_t qmin = g.dn ? 0u : 1u;
    unsigned long long my_count = 0, bytes = 0, obytes = 0;   // bytes: 4 per survivor; obytes: output
    unsigned int* work = (unsigned int*)(ctrl + kWork);
    const unsigned long long wbytes = M == kCount ? 0ull : (M == kEnum ? 4ull * q.k : 8ull);

    for (;;) {
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(work, (unsigned)VPW * batch);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (base >= nent) break;
#pragma unroll 1
        for (uint32_t bt = 0; bt < batch; ++bt) {
            const uint32_t ei = base + bt * VPW + (uint32_t)(lane / G);
            if (!__any_sync(0xffffffffu, ei < nent)) break;
            const bool has = ei < nent;
            const uint32_t e = elist ? __ldg(elist + (has ? ei : 0u)) : ea + (has ? ei : 0);
            // this entry's item range, clipped to [t0, t1)
            uint32_t ilo = 0, ihi = 0;
            uint64_t so = 0, obase = 0;
            uint32_t path[J];
            const uint32_t* lb[NLA];   // list cursors (advance)
            uint32_t ln[NLA];          // remaining lengths (| kBmFlag: bitmap row)
            if (has) {
                const uint64_t o0 = offs[e], o1 = offs[e + 1];
                ilo = (uint32_t)((o0 > t0 ? o0 : t0) - o0);
                ihi = (uint32_t)((o1 < t1 ? o1 : t1) - o0);
                so = src_off[e];
                if (M == kWrite && ord_pos) obase = ord_pos[e] - ord_pos[ord_ea];
#pragma unroll
                for (int p = 0; p < J; ++p) path[p] = p >= (int)pmin ? path_s[(size_t)p * W + e] : 0xffffffffu;
#pragma unroll
                for (int x = 0; x < NL; ++x) {
                    const uint64_t off = lst_off[(size_t)x * W + e];
                    ln[x] = lst_len[(size_t)x * W + e];
                    lb[x] = ((ln[x] & kBmFlag) && ln[x] != kSkip ? g.bm : g.col) + off;
                }
            } else {
#pragma unroll
                for (int p = 0; p < J; ++p) path[p] = 0xffffffffu;
#pragma unroll
                for (int x = 0; x < NLA; ++x) { ln[x] = 0; lb[x] = g.col; }
            }
            // candidate source: a CSR list (u32 stride) or an ancestor's children range
            // in the trie (uint2 stride, .x = vertex)
            const bool tsrc = (so & kTrieSrc) != 0;
            // a component root's free list is already degree-filtered
            const bool fsrc = (so & kFreeSrc) != 0;
            // ... or, when the lists did not fit the arena, the identity list [0, n): candidate = item
            const bool isrc = fsrc && (so & kIdSrc) != 0;
            const uint32_t qlo = isrc ? 0u : qmin;      // an identity candidate may have degree 0
            // packed CSR source (degree in the id word) only where a degree filter applies
            const bool pk = !tsrc && !fsrc && g.colx != nullptr && qd > qmin;
            const uint32_t* __restrict__ src = tsrc ? (const uint32_t*)(rsrc + (so & ~kTrieSrc))
                                             : fsrc ? g.fre + (so & ~(kFreeSrc | kIdSrc)) : (pk ? g.colx : g.col) + so;
            const uint32_t ssh = tsrc ? 1u : 0u;
            const uint32_t umask = pk ? kPackMask : 0xffffffffu;
            // an ancestor range already passed deg >= qdeg[a]: no check needed when qdeg[J] <= qdeg[a]
            const bool dload = qd > qlo && !pk && !(fsrc && !isrc) && !(tsrc && qd <= qda);
            const uint32_t nit = (ihi - ilo + G - 1) / G;
            unsigned long long ecnt = 0, run = 0;   // per-entry count (pass A) / ordered-write cursor
            uint32_t nit_max = nit;
            if (VPW > 1) {
#pragma unroll
                for (int o = 16; o >= G; o >>= 1) nit_max = max(nit_max, __shfl_xor_sync(0xffffffffu, nit_max, o));
            }
            // output of one candidate per lane: warp-aggregated slots
            auto emit = [&](bool ok, uint32_t c) {
                if (M == kCount) {
                    my_count += ok ? 1 : 0;
                    ecnt += ok ? 1 : 0;
                } else if (M == kWrite && ord_pos) {
                    // ordered write: the entry's children are contiguous at its exact offset
                    const unsigned seg = (__ballot_sync(0xffffffffu, ok) >> vb) & kGMask;
                    const unsigned long long pos = obase + run + __popc(seg & ((1u << vl) - 1u));
                    run += __popc(seg);
                    if (ok && pos < cap) out_level[pos] = make_uint2(c, (uint32_t)(w0 + e));
                } else {
                    const unsigned m = __ballot_sync(0xffffffffu, ok);
                    const int nsel = __popc(m);
                    unsigned long long pos0 = 0;
                    if (lane == 0 && nsel) pos0 = atomicAdd(ctrl + (M == kWrite ? kCursor : kEnumCursor), (unsigned long long)nsel);
                    pos0 = __shfl_sync(0xffffffffu, pos0, 0);
                    const unsigned long long pos = pos0 + __popc(m & ((1u << lane) - 1u));
                    if (ok && pos < cap) {
                        if (M == kWrite) {
                            out_level[pos] = make_uint2(c, (uint32_t)(w0 + e));
                        } else {
                            uint32_t* row = out_rows + pos * q.k;
#pragma unroll
                            for (int p = 0; p < J; ++p) row[q.S[p]] = path[p];
                            row[q.S[J]] = c;
                        }
                    }
                }
            };
            bool fast = false;
            if constexpr (NL == 0 && M == kCount) fast = !tsrc && !fsrc && fast_last<J>(q, q.bw[J] | (q.bwi[J] << J), qmin);
            if (fast) {
                // |list[ilo, ihi) \ path|: lane vl < J looks for path[vl] (a distinct vertex)
                if (has) {
                    unsigned long long c = vl == 0 ? (unsigned long long)(ihi - ilo) : 0ull;
                    if (count_bytes && vl == 0) bytes += 4ull * (ihi - ilo);   // model: every element survives
                    if (vl < J && ihi > ilo) {
                        uint32_t x = path[0];
#pragma unroll
                        for (int p = 1; p < J; ++p) x = (p == vl) ? path[p] : x;
                        const uint32_t* b0 = src + ilo;
                        uint32_t len = ihi - ilo;
                        while (len > 1) {
                            const uint32_t half = len >> 1;
                            b0 = (__ldg(b0 + half - 1) < x) ? b0 + half : b0;
                            len -= half;
                        }
                        if (__ldg(b0) == x) c -= 1ull;    // u64 wrap: the warp sum is exact
                    }
                    my_count += c;
                    ecnt += c;
                }
            } else if constexpr (NL == 0) {
                // one backward list: it is the source, so the intersection is the list
                // itself and only injectivity + degree remain; two candidates per lane per
                // iteration, loads issued together
#pragma unroll 1
                for (uint32_t it = 0; it < nit_max; it += 2) {
                    const uint32_t i0 = ilo + it * G + vl, i1 = i0 + G;
                    const bool a0 = i0 < ihi, a1 = i1 < ihi;
                    const uint32_t r0 = a0 ? (isrc ? i0 : __ldg(src + ((size_t)i0 << ssh))) : 0u;
                    const uint32_t r1 = a1 ? (isrc ? i1 : __ldg(src + ((size_t)i1 << ssh))) : 0u;
                    const uint32_t c0 = r0 & umask, c1 = r1 & umask;
                    bool k0 = a0, k1 = a1;
#pragma unroll
                    for (int p = 0; p < J; ++p) { k0 = k0 && (path[p] != c0); k1 = k1 && (path[p] != c1); }
                    if (qdi) {
                        k0 = k0 && __ldg(g.deg + g.dn + c0) >= qdi;
                        k1 = k1 && __ldg(g.deg + g.dn + c1) >= qdi;
                    }
                    if (qd > qlo) {
                        const uint32_t d0 = pk ? (r0 >> kPackShift) : ((k0 && dload) ? __ldg(g.deg + c0) : 0xffffffffu);
                        const uint32_t d1 = pk ? (r1 >> kPackShift) : ((k1 && dload) ? __ldg(g.deg + c1) : 0xffffffffu);
                        k0 = k0 && d0 >= qd;
                        k1 = k1 && d1 >= qd;
                    }
                    if (count_bytes) {
                        bytes += (a0 ? 4ull : 0ull) + (a1 ? 4ull : 0ull);
                        obytes += (k0 ? wbytes : 0ull) + (k1 ? wbytes : 0ull);
                    }
                    emit(k0, c0);
                    if (it + 1 < nit_max) emit(k1, c1);
                }
            } else {
            for (uint32_t it = 0; it < nit_max; ++it) {
                const uint32_t i = ilo + it * G + vl;
                const bool act = i < ihi;
                const uint32_t raw = act ? __ldg(src + ((size_t)i << ssh)) : 0u;
                const uint32_t c = raw & umask;
                bool inj = act;
#pragma unroll
                for (int p = 0; p < J; ++p) inj = inj && (path[p] != c);      // injectivity
                // independent loads issued together: degree (Def. 5) and every hub-bitmap probe
                const bool pre = count_bytes ? act : inj;
                const uint32_t dg = pk ? (raw >> kPackShift) : ((inj && dload) ? __ldg(g.deg + c) : 0xffffffffu);
                uint32_t bmw[NLA];
#pragma unroll
                for (int x = 0; x < NL; ++x)
                    bmw[x] = (pre && (ln[x] & kBmFlag) && ln[x] != kSkip) ? __ldg(lb[x] + (c >> 5)) : 0xffffffffu;
                bool ok = inj && dg >= qd;                                    // every neighbour has deg >= 1
                if (qdi) ok = ok && __ldg(g.deg + g.dn + c) >= qdi;          // directed: in-degree
                bool inter = count_bytes ? act : ok;
#pragma unroll
                for (int x = 0; x < NL; ++x)                                  // c-intersection (Alg. 2): hubs
                    inter = inter && ((bmw[x] >> (c & 31)) & 1u);
#pragma unroll
                for (int x = 0; x < NL; ++x) {                                // c-intersection: sorted lists
                    const bool pend = inter && !(ln[x] & kBmFlag);
                    const unsigned pw = __ballot_sync(0xffffffffu, pend);
                    if (pw) {
                        uint32_t pos = 0;
                        if (pend) {     // branch-free lower bound from the cursor
                            const uint32_t* b0 = lb[x];
                            uint32_t len = ln[x];
                            while (len > 1) {
                                const uint32_t half = len >> 1;
                                b0 = (__ldg(b0 + half - 1) < c) ? b0 + half : b0;
                                len -= half;
                            }
                            inter = len == 1 && __ldg(b0) == c;
                            pos = (uint32_t)(b0 - lb[x]);
                        }
                        // candidates ascend with the lane, so the highest pending lane of
                        // the virtual warp holds the furthest safe cursor position
                        const unsigned pv = (pw >> vb) & kGMask;
                        const int hl = pv ? vb + 31 - __clz(pv) : lane;
                        const uint32_t mpos = __shfl_sync(0xffffffffu, pos, hl);
                        if (pv) { lb[x] += mpos; ln[x] -= mpos; }
                    }
                }
                if (count_bytes) {
                    bytes += inter ? 4ull : 0ull;
                    obytes += inter && ok ? wbytes : 0ull;
                }
                ok = ok && inter;
                emit(ok, c);
            }
            }
            if (M == kCount && ord_cnt) {     // pass A of an ordered level: children per entry
#pragma unroll
                for (int o = G / 2; o >= 1; o >>= 1) ecnt += __shfl_xor_sync(0xffffffffu, ecnt, o);
                if (has && vl == 0) ord_cnt[e] = ecnt;
            }
        }
    }
    if (M == kCount && !ord_cnt) {
        my_count = warp_sum(my_count) * cmul;     // cmul 2: symmetric last level (Reuse::sym)
        if (lane == 0) add_u128(ctrl + kCountLo, my_count);
    }
    if (count_bytes) {
        bytes = warp_sum(bytes);
        obytes = warp_sum(obytes);
        if (lane == 0) {
            atomicAdd(ctrl + kBytesExt, bytes);
            atomicAdd(ctrl + kBytesOut, obytes);
        }
    }
}

// ------------------------------------- §8.d model bytes for the fused kernels
// CUTS_DEBUG_BYTES in k_pairs / k_lr_*: the SURVEY §8.d per-entry model (DESIGN.md
// §5) of the levels these kernels carry, so the instrumented pass runs the same
// kernels as the timed one.  Degree sum of the lists of bw over the trie path of a
// level-`lev` entry (walk `lev`-1 parent hops; path[lev-1] = the entry's vertex).
__device__ __forceinline__ unsigned long long bw_degree_sum(const Graph& g, const Trie& t, uint32_t lev, uint64_t e,
                                                            uint32_t bw) {
    unsigned long long d = 0;
    uint2 cur = t.lv[lev][e];
    for (int p = (int)lev - 1; p >= 0; --p) {
        if ((bw >> p) & 1u) d += __ldg(g.deg + cur.x);
        if (p > 0) cur = t.lv[p][cur.y];
    }
    return d;
}

__device__ __forceinline__ void flush_model_bytes(unsigned long long plan, unsigned long long ext,
                                                  unsigned long long out, unsigned long long need,
                                                  unsigned long long* ctrl) {
    plan = warp_sum(plan); ext = warp_sum(ext); out = warp_sum(out); need = warp_sum(need);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(ctrl + kBytesPlan, plan);
        atomicAdd(ctrl + kBytesExt, ext);
        if (out) atomicAdd(ctrl + kBytesOut, out);
        atomicAdd(ctrl + kBytesNeed, need);
    }
}

// ------------------------------------------- symmetric last level: pair count
// The count-only last level J = k-1 when the level J-1 -> J extension was written
// ordered and the only condition left is adjacency to the entry itself (cliques;
// Reuse::sym): entry e (vertex c_e, parent p) of the level-J chunk has as
// candidates its siblings, the children of p, stored contiguously and ascending;
// sibling c_j is a child of e iff {c_e, c_j} is an edge (the degree filter and
// injectivity are implied: DESIGN.md §7).  Each unordered sibling pair is tested
// once — e tests only the siblings after itself — and the sum is doubled.  No
// plan pass: virtual warps of G lanes take entries straight from the chunk, read
// the sibling range end from the parent's scan slot and test membership in N(c_e)
// by the hub bitmap or a cursor-narrowed binary search (candidates ascend).
//   lv     : the level-J chunk (.x = vertex, .y = index of the parent in level J-1)
//   cpos   : level J-1 window's exclusive scan of child counts; cw0 = that window's
//            start (parent index p -> slot p - cw0); cea = slot of the chunk's first parent
template <int G, bool count_bytes>
__global__ void __launch_bounds__(256, 6) k_pairs(Graph g, const uint2* __restrict__ lv, uint64_t nent,
                                                  const uint64_t* __restrict__ cpos, uint64_t cw0, uint64_t cea,
                                                  unsigned long long* __restrict__ ctrl, uint32_t batch,
                                                  Trie t, uint32_t lev, uint32_t bw) {
    const uint64_t cbase = cpos[cea];
    unsigned long long b_plan = 0, b_ext = 0, b_need = 0;
    constexpr int VPW = 32 / G;
    constexpr unsigned kGMask = G == 32 ? 0xffffffffu : ((1u << G) - 1u);
    const int lane = threadIdx.x & 31;
    const int vl = lane & (G - 1);
    const int vb = lane & ~(G - 1);
    unsigned long long my_count = 0;
    unsigned long long* work = ctrl + kWork;
    for (;;) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(work, (unsigned long long)VPW * batch);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (base >= nent) break;
#pragma unroll 1
        for (uint32_t bt = 0; bt < batch; ++bt) {
            const uint64_t e = base + (uint64_t)bt * VPW + (uint64_t)(lane / G);
            if (!__any_sync(0xffffffffu, e < nent)) break;
            const bool has = e < nent;
            uint32_t v = 0, len = 0;
            uint64_t end = 0;
            const uint32_t* lb = g.col;
            bool bmp = false;
            if (has) {
                const uint2 x = lv[e];
                v = x.x;
                end = cpos[x.y - cw0 + 1] - cbase;
                const uint32_t h = g.hub ? __ldg(g.hub + v) : kNoHub;
                if (h != kNoHub) {
                    bmp = true;
                    lb = g.bm + (uint64_t)h * g.words;
                } else {
                    const uint64_t b = g.row_ptr[v];
                    lb = g.col + b;
                    len = (uint32_t)(g.row_ptr[v + 1] - b);
                }
            }
            const uint32_t nit = has ? (uint32_t)((end - (e + 1) + G - 1) / G) : 0u;
            uint32_t nit_max = nit;
            if (VPW > 1) {
#pragma unroll
                for (int o = 16; o >= G; o >>= 1) nit_max = max(nit_max, __shfl_xor_sync(0xffffffffu, nit_max, o));
            }
            if (count_bytes && has && vl == 0) {   // model: entry + hops + bounds + every backward list
                b_plan += 8ull + 8ull * (lev - 1) + 16ull * __popc(bw);
                b_ext += 4ull * bw_degree_sum(g, t, lev, e, bw);
                b_need += 8ull + 8ull + (bmp ? 4ull : 16ull);
            }
            for (uint32_t it = 0; it < nit_max; ++it) {
                const uint64_t j = e + 1 + (uint64_t)it * G + vl;
                const bool act = has && j < end;
                const uint32_t c = act ? lv[j].x : 0u;
                bool ok = act;
                if (count_bytes && act) b_need += 4ull + 4ull * (bmp ? 1u : (32u - __clz(len)));
                if (bmp && act) ok = (__ldg(lb + (c >> 5)) >> (c & 31)) & 1u;   // hub: one bitmap probe
                const bool pend = act && !bmp;
                const unsigned pw = __ballot_sync(0xffffffffu, pend);
                uint32_t pos = 0;
                if (pend) {          // branch-free lower bound from the cursor
                    const uint32_t* b0 = lb;
                    uint32_t l = len;
                    while (l > 1) {
                        const uint32_t half = l >> 1;
                        b0 = (__ldg(b0 + half - 1) < c) ? b0 + half : b0;
                        l -= half;
                    }
                    ok = len > 0 && __ldg(b0) == c;
                    pos = (uint32_t)(b0 - lb);
                }
                // siblings ascend with the lane: the highest pending lane bounds the cursor
                const unsigned pv = (pw >> vb) & kGMask;
                const int hl = pv ? vb + 31 - __clz(pv) : lane;
                const uint32_t mpos = __shfl_sync(0xffffffffu, pos, hl);
                if (pv) { lb += mpos; len -= mpos; }
                my_count += ok ? 1 : 0;
            }
        }
    }
    my_count = warp_sum(my_count) * 2ull;          // every unordered pair counted once
    if (lane == 0) add_u128(ctrl + kCountLo, my_count);
    // model: 4 B per intersection survivor = per child counted (both ends of each pair)
    if (count_bytes) flush_model_bytes(b_plan, b_ext + (lane == 0 ? 4ull * my_count : 0ull), 0ull, b_need, ctrl);
}

// ------------------------------------------------ local rows (clique tail)
// The last two extension levels of a clique-like tail ("local rows"):
// level-b entries (b = k-2) come in sibling groups S_q (the ordered children of a
// level-(b-1) entry q, contiguous, ascending).  When both remaining extensions only
// add adjacency to the newest vertex (Reuse::sym conditions at b and at b+1), then
//   children(e_i)        = S_q[R_i]            with R_i = {j : S_q[j] in N(S_q[i])}
//   children((e_i, c_j)) = S_q[R_i & R_j]
// so for a group with m <= 64 members the 64-bit rows R_i are all the intersection
// work: |L_{b+1}| += popc(R_i) and the count += sum_{j in R_i} popc(R_i & R_j).
// k_lr_rows tests every unordered sibling pair once (hub bitmap or cursor-narrowed
// binary search, as k_pairs) and sets both bits; k_lr_count does the bit algebra.
// Groups with m > 64 are left to the ordinary pipeline (Reuse::skip_small).
template <int G, bool count_bytes>
__global__ void __launch_bounds__(256, 6) k_lr_rows(Graph g, const uint2* __restrict__ lv, uint64_t nent,
                                                    const uint64_t* __restrict__ cpos, uint64_t cw0, uint64_t cea,
                                                    unsigned long long* __restrict__ R,
                                                    unsigned long long* __restrict__ ctrl, uint32_t batch) {
    unsigned long long b_need = 0;
    constexpr int VPW = 32 / G;
    constexpr unsigned kGMask = G == 32 ? 0xffffffffu : ((1u << G) - 1u);
    const uint64_t cbase = cpos[cea];
    const int lane = threadIdx.x & 31;
    const int vl = lane & (G - 1);
    const int vb = lane & ~(G - 1);
    unsigned long long large = 0;
    unsigned long long* work = ctrl + kWork;
    for (;;) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(work, (unsigned long long)VPW * batch);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (base >= nent) break;
#pragma unroll 1
        for (uint32_t bt = 0; bt < batch; ++bt) {
            const uint64_t e = base + (uint64_t)bt * VPW + (uint64_t)(lane / G);
            if (!__any_sync(0xffffffffu, e < nent)) break;
            bool has = e < nent;
            uint32_t v = 0, len = 0;
            uint64_t g0 = 0, end = 0;
            const uint32_t* lb = g.col;
            bool bmp = false;
            if (has) {
                const uint2 x = lv[e];
                v = x.x;
                g0 = cpos[x.y - cw0] - cbase;
                end = cpos[x.y - cw0 + 1] - cbase;
                if (end - g0 > 64) {             // k_lr_group or (> kLrMaxM) the ordinary pipeline
                    if (vl == 0 && end - g0 > (uint64_t)kLrMaxM) large += 1;
                    has = false;
                } else {
                    const uint32_t h = g.hub ? __ldg(g.hub + v) : kNoHub;
                    if (h != kNoHub) {
                        bmp = true;
                        lb = g.bm + (uint64_t)h * g.words;
                    } else {
                        const uint64_t b = g.row_ptr[v];
                        lb = g.col + b;
                        len = (uint32_t)(g.row_ptr[v + 1] - b);
                    }
                }
            }
            const uint32_t nit = has ? (uint32_t)((end - (e + 1) + G - 1) / G) : 0u;
            uint32_t nit_max = nit;
            if (VPW > 1) {
#pragma unroll
                for (int o = 16; o >= G; o >>= 1) nit_max = max(nit_max, __shfl_xor_sync(0xffffffffu, nit_max, o));
            }
            unsigned long long row = 0;
            if (count_bytes && has && vl == 0) b_need += 8ull + 8ull + (bmp ? 4ull : 16ull) + 8ull;   // + the row
            for (uint32_t it = 0; it < nit_max; ++it) {
                const uint64_t j = e + 1 + (uint64_t)it * G + vl;
                const bool act = has && j < end;
                const uint32_t c = act ? lv[j].x : 0u;
                bool ok = act;
                if (count_bytes && act) b_need += 4ull + 4ull * (bmp ? 1u : (32u - __clz(len)));
                if (bmp && act) ok = (__ldg(lb + (c >> 5)) >> (c & 31)) & 1u;
                const bool pend = act && !bmp;
                const unsigned pw = __ballot_sync(0xffffffffu, pend);
                uint32_t pos = 0;
                if (pend) {
                    const uint32_t* b0 = lb;
                    uint32_t l = len;
                    while (l > 1) {
                        const uint32_t half = l >> 1;
                        b0 = (__ldg(b0 + half - 1) < c) ? b0 + half : b0;
                        l -= half;
                    }
                    ok = len > 0 && __ldg(b0) == c;
                    pos = (uint32_t)(b0 - lb);
                }
                const unsigned pv = (pw >> vb) & kGMask;
                const int hl = pv ? vb + 31 - __clz(pv) : lane;
                const uint32_t mpos = __shfl_sync(0xffffffffu, pos, hl);
                if (pv) { lb += mpos; len -= mpos; }
                if (ok) {                          // the pair {i, j}: bit j of R_i and bit i of R_j
                    row |= 1ull << (j - g0);
                    atomicOr(R + j, 1ull << (e - g0));
                }
            }
#pragma unroll
            for (int o = G / 2; o >= 1; o >>= 1) row |= __shfl_xor_sync(0xffffffffu, row, o);
            if (has && vl == 0 && row) atomicOr(R + e, row);
        }
    }
    large = warp_sum(large);
    if (lane == 0 && large) atomicAdd(ctrl + kLrLarge, large);
    if (count_bytes) flush_model_bytes(0, 0, 0, b_need, ctrl);
}

// Mid-size groups (64 < m <= kLrMaxM): one CTA per group builds the m x m sibling
// adjacency in shared memory (each unordered pair tested once by a warp: hub bitmap or
// cursor-narrowed binary search, both bits set), then the same bit algebra as
// k_lr_count: |L_{b+1}| += popc(A_i), count += sum_{j in A_i} popc(A_i & A_j).
// CTAs pull parent slots (groups) from a work counter.
template <bool count_bytes>
__global__ void __launch_bounds__(256) k_lr_group(Graph g, const uint2* __restrict__ lv,
                                                  const uint64_t* __restrict__ cpos, uint64_t cea, uint64_t ceb,
                                                  unsigned long long* __restrict__ ctrl, Trie t, uint32_t lev,
                                                  uint32_t bw_b, uint32_t bw_c) {
    __shared__ uint32_t S[kLrMaxM];
    __shared__ uint32_t A[kLrMaxM][kLrWords + 1];   // odd row stride: lanes on distinct rows hit distinct banks
    __shared__ uint64_t s_q;
    __shared__ uint32_t s_n, s_list[kLrBatch];
    unsigned long long b_plan = 0, b_ext = 0, b_out = 0, b_need = 0;
    const uint64_t cbase = cpos[cea];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    unsigned long long lvl = 0, cnt = 0;
    unsigned long long* work = ctrl + kLrWork;
    for (;;) {
        // a batch of kLrBatch parent slots per CTA: one thread tests each slot's group
        // size (coalesced cpos reads) and the mid-size groups are listed in shared memory
        __syncthreads();
        if (threadIdx.x == 0) { s_q = cea + atomicAdd(work, (unsigned long long)kLrBatch); s_n = 0; }
        __syncthreads();
        const uint64_t qb = s_q;
        if (qb >= ceb) break;
        for (uint32_t x = threadIdx.x; x < (uint32_t)kLrBatch; x += blockDim.x) {
            const uint64_t q = qb + x;
            if (q < ceb) {
                const uint64_t m = cpos[q + 1] - cpos[q];
                if (m > 64 && m <= (uint64_t)kLrMaxM) s_list[atomicAdd(&s_n, 1u)] = x;
            }
        }
        __syncthreads();
        const uint32_t nlist = s_n;
        for (uint32_t li = 0; li < nlist; ++li) {
        __syncthreads();
        const uint64_t q = qb + s_list[li];
        const uint64_t g0 = cpos[q] - cbase, g1 = cpos[q + 1] - cbase;
        const uint32_t m = (uint32_t)(g1 - g0);
        const uint32_t W = (m + 31) / 32;
        for (uint32_t i = threadIdx.x; i < m; i += blockDim.x) S[i] = lv[g0 + i].x;
        for (uint32_t i = threadIdx.x; i < m * (kLrWords + 1); i += blockDim.x) (&A[0][0])[i] = 0u;
        __syncthreads();
        for (uint32_t i = warp; i + 1 < m; i += nw) {            // row i tests the members after it
            const uint32_t v = S[i];
            const uint32_t h = g.hub ? __ldg(g.hub + v) : kNoHub;
            const uint32_t* lb;
            uint32_t len = 0;
            if (h != kNoHub) lb = g.bm + (uint64_t)h * g.words;
            else { const uint64_t b = g.row_ptr[v]; lb = g.col + b; len = (uint32_t)(g.row_ptr[v + 1] - b); }
            for (uint32_t j0 = i + 1; j0 < m; j0 += 32) {
                const uint32_t j = j0 + lane;
                const bool act = j < m;
                const uint32_t c = act ? S[j] : 0u;
                bool ok = false;
                if (count_bytes && act) b_need += 4ull * (h != kNoHub ? 1u : (32u - __clz(len)));
                if (h != kNoHub) {
                    ok = act && ((__ldg(lb + (c >> 5)) >> (c & 31)) & 1u);
                } else {
                    uint32_t pos = 0;
                    if (act) {
                        const uint32_t* b0 = lb;
                        uint32_t l = len;
                        while (l > 1) {
                            const uint32_t half = l >> 1;
                            b0 = (__ldg(b0 + half - 1) < c) ? b0 + half : b0;
                            l -= half;
                        }
                        ok = len > 0 && __ldg(b0) == c;
                        pos = (uint32_t)(b0 - lb);
                    }
                    const unsigned pw = __ballot_sync(0xffffffffu, act);
                    const uint32_t mpos = __shfl_sync(0xffffffffu, pos, 31 - __clz(pw));
                    lb += mpos;
                    len -= mpos;
                }
                if (ok) {
                    atomicOr(&A[i][j >> 5], 1u << (j & 31));
                    atomicOr(&A[j][i >> 5], 1u << (i & 31));
                }
            }
        }
        __syncthreads();
        for (uint32_t i = warp; i < m; i += nw) {                // bit algebra, a warp per row
            uint32_t ri[kLrWords];
#pragma unroll
            for (int w = 0; w < kLrWords; ++w) ri[w] = (uint32_t)w < W ? A[i][w] : 0u;
            unsigned long long pi = 0;
#pragma unroll
            for (int w = 0; w < kLrWords; ++w) pi += __popc(ri[w]);
            if (lane == 0) lvl += pi;
            unsigned long long db = 0;
            if (count_bytes) {        // the members share the parent's path: walk from member i
                db = bw_degree_sum(g, t, lev, g0 + i, bw_b);
                if (lane == 0) {
                    b_plan += 8ull + 8ull * (lev - 1) + 16ull * __popc(bw_b) + pi * (8ull + 8ull * lev + 16ull * __popc(bw_c));
                    b_ext += 4ull * db + 4ull * pi;
                    b_out += 8ull * pi;
                    b_need += 8ull + 8ull + 16ull;
                }
            }
            for (uint32_t j = lane; j < m; j += 32) {             // lane takes the members j in row i
                if (!((A[i][j >> 5] >> (j & 31)) & 1u)) continue;   // (smem: no dynamic register index)
                uint32_t c = 0;
#pragma unroll
                for (int w = 0; w < kLrWords; ++w) c += (uint32_t)w < W ? __popc(ri[w] & A[j][w]) : 0u;
                cnt += c;
                if (count_bytes) b_ext += 4ull * (db + __ldg(g.deg + S[j])) + 4ull * c;
            }
        }
        }
    }
    lvl = warp_sum(lvl);
    cnt = warp_sum(cnt);
    if (lane == 0) {
        if (lvl) atomicAdd(ctrl + kLrLevel, lvl);
        add_u128(ctrl + kCountLo, cnt);
    }
    if (count_bytes) flush_model_bytes(b_plan, b_ext, b_out, b_need, ctrl);
}

// thread per level-b entry of a small group: |L_{b+1}| and the count from the rows
// With count_bytes it also adds the §8.d model of both carried levels: the level-b
// entry's extension (lists of bw_b, survivors, children written) and every child's
// count-only extension (lists of bw_b plus the child's own, survivors).
template <bool count_bytes>
__global__ void k_lr_count(Graph g, const uint2* __restrict__ lv, uint64_t nent, const uint64_t* __restrict__ cpos,
                           uint64_t cw0, uint64_t cea, const unsigned long long* __restrict__ R,
                           unsigned long long* __restrict__ ctrl, Trie t, uint32_t lev, uint32_t bw_b,
                           uint32_t bw_c) {
    const uint64_t cbase = cpos[cea];
    unsigned long long lvl = 0, cnt = 0, b_plan = 0, b_ext = 0, b_out = 0, b_need = 0;
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nent;
         e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t p = lv[e].y;
        const uint64_t g0 = cpos[p - cw0] - cbase, g1 = cpos[p - cw0 + 1] - cbase;
        if (g1 - g0 > 64) continue;
        const unsigned long long r = R[e];
        lvl += __popcll(r);
        unsigned long long db = 0;
        if (count_bytes) {
            db = bw_degree_sum(g, t, lev, e, bw_b);
            b_plan += 8ull + 8ull * (lev - 1) + 16ull * __popc(bw_b) +
                      (unsigned long long)__popcll(r) * (8ull + 8ull * lev + 16ull * __popc(bw_c));
            b_ext += 4ull * db + 4ull * __popcll(r);
            b_out += 8ull * __popcll(r);
            b_need += 8ull + 8ull + 16ull + 8ull;
        }
        for (unsigned long long b = r; b; b &= b - 1) {
            const uint64_t j = g0 + __ffsll((long long)b) - 1;
            const unsigned long long s2 = __popcll(r & R[j]);
            cnt += s2;
            if (count_bytes) {
                b_ext += 4ull * (db + __ldg(g.deg + lv[j].x)) + 4ull * s2;
                b_need += 8ull;
            }
        }
    }
    lvl = warp_sum(lvl);
    cnt = warp_sum(cnt);
    if ((threadIdx.x & 31) == 0) {
        if (lvl) atomicAdd(ctrl + kLrLevel, lvl);
        add_u128(ctrl + kCountLo, cnt);
    }
    if (count_bytes) flush_model_bytes(b_plan, b_ext, b_out, b_need, ctrl);
}

// ------------------------------------------------ deep local rows (clique tail)
// DESIGN.md §7 "deep local rows": the local-rows idea one level higher.  When the
// last THREE extensions of a count-only query only add adjacency to the newest vertex
// (Reuse::sym conditions at b, b+1, b+2 with b = k-3), a level-b sibling group
// G = (G[0] < ... < G[m-1]) (the ordered children of one level-(b-1) entry) and its
// adjacency rows A_t = {s : G[s] in N(G[t])} carry all three:
//   children(e_t)            = G[A_t]                       -> level b+1, WRITTEN (trie)
//   children((e_t, G[s]))    = G[A_t & A_s]                 -> |L_{b+2}| (fused)
//   children((e_t, G[s], G[l])) = G[A_t & A_s & A_l]        -> the count
// Rows are W = ceil(m/64) u64 words; every unordered pair of G is tested once (hub
// bitmap or cursor-narrowed binary search), so a group costs m^2/2 membership tests
// instead of the m_child^2/2 of every child group below it.  Groups of more than
// kDlrMaxM members are left to the windowed pipeline (Reuse::skip_small).
struct Dlr {
    const uint2* lv;            // level-b chunk (.x vertex, .y parent index in level b-1)
    uint64_t n;                 // entries of the chunk
    const uint64_t* cpos;       // level b-1 window: exclusive scan of child counts
    uint64_t w0, ea, eb;        // window start; parent slots [ea, eb) own the chunk (window-relative)
    const uint64_t* roff;       // row word offset of each parent slot's group (slot - ea)
    unsigned long long* R;      // rows
    unsigned long long* desc;   // per entry: rb | te << 40 | m << 51 (k_dlr_desc); ~0: group too large
};

struct DlrGrp {
    uint64_t g0;                // first member (chunk index)
    uint64_t rb;                // first row word
    uint32_t m, W;
};

__device__ __forceinline__ DlrGrp dlr_group(const Dlr& a, uint64_t e) {
    const unsigned long long d = a.desc[e];
    DlrGrp gr;
    if (d == ~0ull) { gr.g0 = e; gr.rb = 0; gr.m = kDlrMaxM + 1; gr.W = 0; return gr; }
    const uint32_t te = (uint32_t)(d >> 40) & 0x7ffu;
    gr.g0 = e - te;
    gr.rb = d & ((1ull << 40) - 1);
    gr.m = (uint32_t)(d >> 51) & 0x7ffu;
    gr.W = (gr.m + 63) / 64;
    return gr;
}

// per entry of the level-b chunk: its group's row base, its index in the group and the
// group size, packed (one 8-byte load per entry for every later kernel)
__global__ void k_dlr_desc(Dlr a) {
    const uint64_t c0 = a.cpos[a.ea];
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < a.n; e += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t q = (uint64_t)a.lv[e].y - a.w0;
        const uint64_t q0 = a.cpos[q], m = a.cpos[q + 1] - q0;
        a.desc[e] = m > (uint64_t)kDlrMaxM ? ~0ull
                                           : (a.roff[q - a.ea] | ((e - (q0 - c0)) << 40) | (m << 51));
    }
}

// CUB select predicate: parent slot x (window-relative, from ea) owns a group of 129..1024
// members (k_dlr_tail_cta's work list)
struct DlrIsWide {
    const uint64_t* cpos;
    uint64_t ea;
    __host__ __device__ bool operator()(const uint32_t& x) const {
        const uint64_t m = cpos[ea + x + 1] - cpos[ea + x];
        return m > 128 && m <= (uint64_t)kDlrMaxM;
    }
};

// ... a group with 65..128 members (two row words): k_dlr_tail_warp<2>'s work list
struct DlrIsMid {
    const uint64_t* cpos;
    uint64_t ea;
    __host__ __device__ bool operator()(const uint32_t& x) const {
        const uint64_t m = cpos[ea + x + 1] - cpos[ea + x];
        return m > 64 && m <= 128;
    }
};

// ... and a group with 2..64 members (one row word): k_dlr_tail_narrow's work list
struct DlrIsNarrow {
    const uint64_t* cpos;
    uint64_t ea;
    __host__ __device__ bool operator()(const uint32_t& x) const {
        const uint64_t m = cpos[ea + x + 1] - cpos[ea + x];
        return m >= 2 && m <= 64;
    }
};

// per parent slot: row words of its group (0 when it is left to the windowed pipeline)
__global__ void k_dlr_layout(Dlr a, uint64_t* __restrict__ rw, unsigned long long* __restrict__ ctrl) {
    unsigned long long large = 0;
    const uint64_t ng = a.eb - a.ea;
    for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x <= ng; x += (uint64_t)gridDim.x * blockDim.x) {
        if (x == ng) { rw[ng] = 0; continue; }
        const uint64_t m = a.cpos[a.ea + x + 1] - a.cpos[a.ea + x];
        rw[x] = m <= (uint64_t)kDlrMaxM ? ((m * ((m + 63) / 64) + 1) & ~1ull) : 0ull;   // even: 16-B aligned blocks
        if (m > (uint64_t)kDlrMaxM) large += m;
    }
    large = warp_sum(large);
    if ((threadIdx.x & 31) == 0 && large) atomicAdd(ctrl + kDlrLarge, large);
}

// Rows: a virtual warp of G lanes per entry t tests the members after it, in G-aligned
// blocks of the group so the block's ballot is one aligned G-bit piece of row t (one
// atomicOr); each hit also sets bit t of the other member's row.
template <int G, bool count_bytes>
__global__ void __launch_bounds__(256, 6) k_dlr_rows(Graph g, Dlr a, unsigned long long* __restrict__ ctrl,
                                                     uint32_t batch) {
    unsigned long long b_need = 0;
    constexpr int VPW = 32 / G;
    constexpr unsigned kGMask = G == 32 ? 0xffffffffu : ((1u << G) - 1u);
    const int lane = threadIdx.x & 31;
    const int vl = lane & (G - 1);
    const int vb = lane & ~(G - 1);
    unsigned long long* work = ctrl + kDlrWork;
    uint32_t* R32 = (uint32_t*)a.R;
    for (;;) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(work, (unsigned long long)VPW * batch);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (base >= a.n) break;
#pragma unroll 1
        for (uint32_t bt = 0; bt < batch; ++bt) {
            const uint64_t e = base + (uint64_t)bt * VPW + (uint64_t)(lane / G);
            if (!__any_sync(0xffffffffu, e < a.n)) break;
            bool has = e < a.n;
            uint32_t len = 0, te = 0, jb = 0, m = 0, W = 0;
            uint64_t g0 = 0, rb = 0;
            const uint32_t* lb = g.col;
            bool bmp = false;
            uint32_t hrow = 0;
            if (has) {
                const DlrGrp gr = dlr_group(a, e);
                g0 = gr.g0; m = gr.m; W = gr.W; rb = gr.rb;
                te = (uint32_t)(e - g0);
                has = m >= 2 && m <= (uint32_t)kDlrMaxM && te + 1 < m;
                if (has) {
                    jb = (te + 1) & ~(uint32_t)(G - 1);
                    const uint32_t v = a.lv[e].x;
                    const uint32_t h = g.hub ? __ldg(g.hub + v) : kNoHub;
                    if (h != kNoHub) {
                        bmp = true;
                        hrow = h;
                    } else {
                        const uint64_t b = g.row_ptr[v];
                        lb = g.col + b;
                        len = (uint32_t)(g.row_ptr[v + 1] - b);
                    }
                }
            }
            const uint32_t nit = has ? (m - jb + G - 1) / G : 0u;
            uint32_t nit_max = nit;
            if (VPW > 1) {
#pragma unroll
                for (int o = 16; o >= G; o >>= 1) nit_max = max(nit_max, __shfl_xor_sync(0xffffffffu, nit_max, o));
            }
            if (count_bytes && has && vl == 0) b_need += 8ull + 16ull + (bmp ? 4ull : 16ull);
            uint32_t* row_e = R32 + 2 * (rb + (uint64_t)te * W);
            for (uint32_t it = 0; it < nit_max; ++it) {
                const uint32_t jj = jb + it * G + vl;
                const bool act = has && jj > te && jj < m;
                const uint32_t c = act ? a.lv[g0 + jj].x : 0u;
                bool ok = act;
                if (count_bytes && act) b_need += 4ull + 4ull * (bmp ? 1u : (32u - __clz(len)));
                if (bmp && act) ok = hub_probe(g, hrow, c);
                const bool pend = act && !bmp;
                const unsigned pw = __ballot_sync(0xffffffffu, pend);
                uint32_t pos = 0;
                if (pend) {
                    const uint32_t* b0 = lb;
                    uint32_t l = len;
                    while (l > 1) {
                        const uint32_t half = l >> 1;
                        b0 = (__ldg(b0 + half - 1) < c) ? b0 + half : b0;
                        l -= half;
                    }
                    ok = len > 0 && __ldg(b0) == c;
                    pos = (uint32_t)(b0 - lb);
                }
                const unsigned pv = (pw >> vb) & kGMask;
                const int hl = pv ? vb + 31 - __clz(pv) : lane;
                const uint32_t mpos = __shfl_sync(0xffffffffu, pos, hl);
                if (pv) { lb += mpos; len -= mpos; }
                const unsigned seg = (__ballot_sync(0xffffffffu, ok) >> vb) & kGMask;
                if (ok) atomicOr(R32 + 2 * (rb + (uint64_t)jj * W) + (te >> 5), 1u << (te & 31));
                if (vl == 0 && seg) {
                    const uint32_t j0 = jb + it * G;
                    atomicOr(row_e + (j0 >> 5), seg << (j0 & 31));
                }
            }
        }
    }
    if (count_bytes) flush_model_bytes(0, 0, 0, b_need, ctrl);
}

// children per entry (0 outside the eligible groups); with count_bytes the §8.d model
// of the level-b -> b+1 extension these rows stand for
template <bool count_bytes>
__global__ void k_dlr_counts(Graph g, Trie t, Dlr a, uint64_t* __restrict__ cnt, unsigned long long* __restrict__ ctrl,
                             uint32_t lev, uint32_t bw_b) {
    unsigned long long b_plan = 0, b_ext = 0, b_out = 0, b_need = 0;
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e <= a.n; e += (uint64_t)gridDim.x * blockDim.x) {
        if (e == a.n) { cnt[e] = 0; continue; }
        const DlrGrp gr = dlr_group(a, e);
        uint64_t c = 0;
        if (gr.m <= (uint32_t)kDlrMaxM) {
            const unsigned long long* r = a.R + gr.rb + (e - gr.g0) * gr.W;
            for (uint32_t w = 0; w < gr.W; ++w) c += __popcll(r[w]);
            if (count_bytes) {
                b_plan += 8ull + 8ull * (lev - 1) + 16ull * __popc(bw_b);
                b_ext += 4ull * bw_degree_sum(g, t, lev, e, bw_b) + 4ull * c;
                b_out += 8ull * c;
                b_need += 8ull * gr.W + 8ull;
            }
        }
        cnt[e] = c;
    }
    if (count_bytes) flush_model_bytes(b_plan, b_ext, b_out, b_need, ctrl);
}

// Where entry e's children sit in the written level-(b+1) chunk (entries [e0, e1)).
// Plain: cpos[e] - cpos[e0].  Split (with k_dlr_tail_cta): the children of narrow-group
// entries (W = 1) first, in entry order, then those of wide-group entries — each
// entry's children still contiguous and ascending — so the warp-queue tail reads only
// [0, nn) and the CTA tail only [nn, size).  cposn = scan of the narrow entries' child
// counts; the wide scan is cpos - cposn.
struct DlrOut {
    const uint64_t* cpos;
    const uint64_t* cposn;            // nullptr: plain layout
    uint64_t e0;
    uint64_t nn;                      // narrow children in the chunk
};
__device__ __forceinline__ uint64_t dlr_child_off(const DlrOut& L, uint64_t e, bool wide) {
    if (!L.cposn) return L.cpos[e] - L.cpos[L.e0];
    if (!wide) return L.cposn[e] - L.cposn[L.e0];
    return L.nn + (L.cpos[e] - L.cposn[e]) - (L.cpos[L.e0] - L.cposn[L.e0]);
}

// narrow-group entries' child counts (the split layout's first scan)
__global__ void k_dlr_narrow(Dlr a, const uint64_t* __restrict__ cnt, uint64_t* __restrict__ cntn) {
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e <= a.n; e += (uint64_t)gridDim.x * blockDim.x) {
        if (e == a.n) { cntn[e] = 0; continue; }
        const unsigned long long d = a.desc[e];
        const uint32_t m = d == ~0ull ? 0u : (uint32_t)(d >> 51) & 0x7ffu;
        cntn[e] = (m > 0 && m <= 64) ? cnt[e] : 0ull;
    }
}

// level b+1 written from the rows: entry e's children G[A_e] at its exact offset
// (ascending, the ordered layout every level of the trie keeps).  A half-warp per entry
// (two entries in flight per warp): lane i of the half owns member 16h+i of each 16-bit
// slice h of the row, ranks come from a popcount of the slice below it, so the member
// reads and the children stores are both coalesced.
__global__ void __launch_bounds__(256) k_dlr_write(Dlr a, DlrOut L, uint64_t e1, uint2* __restrict__ out) {
    const int lane = threadIdx.x & 31, hl = lane & 15;
    const uint64_t nh = ((uint64_t)gridDim.x * blockDim.x) >> 4;
    for (uint64_t e = L.e0 + (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 4); e < e1; e += nh) {
        const unsigned long long d = __ldg(a.desc + e);
        if (d == ~0ull) continue;                                    // half-warp-uniform
        const uint32_t te = (uint32_t)(d >> 40) & 0x7ffu, m = (uint32_t)(d >> 51) & 0x7ffu;
        uint64_t o = dlr_child_off(L, e, m > 64);
        const uint64_t g0 = e - te;
        const uint32_t W = (m + 63) / 64;
        const unsigned long long* r = a.R + (d & ((1ull << 40) - 1)) + (uint64_t)te * W;
        for (uint32_t w = 0; w < W; ++w) {
            const unsigned long long x = __ldg(r + w);
            // the four 16-bit slices of the word: member loads issued together, then the stores
            uint32_t v[4];
#pragma unroll
            for (int h = 0; h < 4; ++h) {
                const bool bit = (x >> (16 * h + hl)) & 1ull;
                v[h] = bit ? __ldg(&a.lv[g0 + 64u * w + 16u * h + hl].x) : 0u;
            }
#pragma unroll
            for (int h = 0; h < 4; ++h) {
                const uint32_t xs = (uint32_t)(x >> (16 * h)) & 0xffffu;
                if ((xs >> hl) & 1u) out[o + __popc(xs & ((1u << hl) - 1u))] = make_uint2(v[h], (uint32_t)e);
                o += __popc(xs);
            }
        }
    }
}

// index of the rank-th set bit (0-based) of a W-word row
__device__ __forceinline__ uint32_t dlr_select(const unsigned long long* r, uint32_t W, uint32_t rank) {
    for (uint32_t w = 0; w < W; ++w) {
        const unsigned long long x = r[w];
        const uint32_t pc = (uint32_t)__popcll(x);
        if (rank < pc) {
            const uint32_t lo = (uint32_t)x, plo = (uint32_t)__popc(lo);
            if (rank < plo) return 64u * w + (uint32_t)__fns(lo, 0, (int)rank + 1);
            return 64u * w + 32u + (uint32_t)__fns((uint32_t)(x >> 32), 0, (int)(rank - plo) + 1);
        }
        rank -= pc;
    }
    return 0xffffffffu;
}

// bits strictly above position p in word w of a row
__device__ __forceinline__ unsigned long long dlr_above(uint32_t p, uint32_t w) {
    const uint32_t pw = p >> 6;
    if (w < pw) return 0ull;
    if (w > pw) return ~0ull;
    return (p & 63u) == 63u ? 0ull : (~0ull << ((p & 63u) + 1u));
}

// The tail counts by symmetry.  The four positions b-1 .. b+2 = k-1 are pairwise adjacent
// in Q with the same backward set outside (the Reuse::sym conditions), so the
// completions of a group are exactly the ordered 4-cliques (G[t], G[s], G[l], G[u]) of
// its adjacency: |L_{b+2}| gets 6 x (triangles t < s < l) and the count 24 x (4-cliques
// t < s < l < u).  The level-(b+1) entry (e_t, G[s]) with t < s holds the ones whose
// two smallest members are t, s: x = A_t & A_s & {> s}, triangles += |x|,
// 4-cliques += sum_{l in x} |x & {> l} & A_l|; an entry with t > s holds none.
// WM: x held in registers for rows of up to WM words (0: re-read from the rows).
template <int WM>
__device__ __forceinline__ void dlr_tail_one(const unsigned long long* __restrict__ Rt,
                                             const unsigned long long* __restrict__ Rs,
                                             const unsigned long long* __restrict__ Rg, uint32_t W, uint32_t s,
                                             unsigned long long& tri, unsigned long long& k4) {
    if constexpr (WM > 0) {
        unsigned long long x[WM];
#pragma unroll
        for (int w = 0; w < WM; ++w) x[w] = (uint32_t)w < W ? (Rt[w] & Rs[w] & dlr_above(s, (uint32_t)w)) : 0ull;
#pragma unroll
        for (int w = 0; w < WM; ++w) {
            tri += __popcll(x[w]);
            for (unsigned long long y = x[w]; y;) {
                const uint32_t l = 64u * w + (uint32_t)(__ffsll((long long)y) - 1);
                y &= y - 1;                                   // the members of x above l in word w
                const unsigned long long* Rl = Rg + (uint64_t)l * W;
                unsigned long long c = __popcll(y & Rl[w]);
#pragma unroll
                for (int v = w + 1; v < WM; ++v) c += (uint32_t)v < W ? __popcll(x[v] & Rl[v]) : 0ull;
                k4 += c;
            }
        }
    } else {
        for (uint32_t w = s >> 6; w < W; ++w) {
            const unsigned long long xw = Rt[w] & Rs[w] & dlr_above(s, w);
            tri += __popcll(xw);
            for (unsigned long long y = xw; y;) {
                const uint32_t l = 64u * w + (uint32_t)(__ffsll((long long)y) - 1);
                y &= y - 1;
                const unsigned long long* Rl = Rg + (uint64_t)l * W;
                unsigned long long c = __popcll(y & Rl[w]);
                for (uint32_t v = w + 1; v < W; ++v) c += __popcll(Rt[v] & Rs[v] & Rl[v]);
                k4 += c;
            }
        }
    }
}

__device__ __forceinline__ void dlr_tail_item(const unsigned long long* __restrict__ R, unsigned long long rb,
                                              uint32_t pk, unsigned long long& tri, unsigned long long& k4) {
    const uint32_t te = pk & 0x7ffu, s = (pk >> 11) & 0x7ffu, W = pk >> 22;
    const unsigned long long* Rg = R + rb;
    const unsigned long long* Rt = Rg + (uint64_t)te * W;
    const unsigned long long* Rs = Rg + (uint64_t)s * W;
    if (W == 1) dlr_tail_one<1>(Rt, Rs, Rg, 1, s, tri, k4);
    else if (W == 2) dlr_tail_one<2>(Rt, Rs, Rg, 2, s, tri, k4);
    else if (W <= 4) dlr_tail_one<4>(Rt, Rs, Rg, W, s, tri, k4);
    else dlr_tail_one<0>(Rt, Rs, Rg, W, s, tri, k4);
}

// bit position of the rank-th (0-based) set bit of y (rank < popc(y))
__device__ __forceinline__ uint32_t dlr_fns64(unsigned long long y, uint32_t rank) {
    const uint32_t lo = (uint32_t)y, plo = (uint32_t)__popc(lo);
    return rank < plo ? (uint32_t)__fns(lo, 0, (int)rank + 1) : 32u + (uint32_t)__fns((uint32_t)(y >> 32), 0, (int)(rank - plo) + 1);
}

// Members l of x = A_t & A_s & {> s} with ranks [r0, r0 + kDlrRun) in ascending order (fewer
// if x runs out): k4 += |x & {> l} & A_l| for each — one split work item of the tail.
// WM: x in registers for rows of up to WM words (0: re-read from the rows).
constexpr uint32_t kDlrRun = 8;
template <int WM>
__device__ __forceinline__ void dlr_run(const unsigned long long* __restrict__ Rg, uint32_t te, uint32_t s, uint32_t W,
                                        uint32_t r0, unsigned long long& k4) {
    const unsigned long long* Rt = Rg + (uint64_t)te * W;
    const unsigned long long* Rs = Rg + (uint64_t)s * W;
    uint32_t rem = kDlrRun, skip = r0;
    if constexpr (WM > 0) {
        unsigned long long x[WM];
#pragma unroll
        for (int w = 0; w < WM; ++w) x[w] = (uint32_t)w < W ? (Rt[w] & Rs[w] & dlr_above(s, (uint32_t)w)) : 0ull;
#pragma unroll
        for (int w = 0; w < WM; ++w) {
            unsigned long long y = x[w];
            const uint32_t pc = (uint32_t)__popcll(y);
            if (rem == 0 || skip >= pc) { skip -= min(skip, pc); continue; }
            if (skip) {                                       // drop the members of lower rank
                const uint32_t p = dlr_fns64(y, skip - 1);
                y &= p == 63u ? 0ull : (~0ull << (p + 1u));
                skip = 0;
            }
            while (y && rem) {
                const uint32_t l = 64u * w + (uint32_t)(__ffsll((long long)y) - 1);
                y &= y - 1;                                   // x's members above l in word w
                --rem;
                const unsigned long long* Rl = Rg + (uint64_t)l * W;
                unsigned long long c = __popcll(y & Rl[w]);
#pragma unroll
                for (int v = w + 1; v < WM; ++v) c += (uint32_t)v < W ? __popcll(x[v] & Rl[v]) : 0ull;
                k4 += c;
            }
        }
    } else {
        for (uint32_t w = s >> 6; w < W && rem; ++w) {
            unsigned long long y = Rt[w] & Rs[w] & dlr_above(s, w);
            const uint32_t pc = (uint32_t)__popcll(y);
            if (skip >= pc) { skip -= pc; continue; }
            if (skip) {
                const uint32_t p = dlr_fns64(y, skip - 1);
                y &= p == 63u ? 0ull : (~0ull << (p + 1u));
                skip = 0;
            }
            while (y && rem) {
                const uint32_t l = 64u * w + (uint32_t)(__ffsll((long long)y) - 1);
                y &= y - 1;
                --rem;
                const unsigned long long* Rl = Rg + (uint64_t)l * W;
                unsigned long long c = __popcll(y & Rl[w]);
                for (uint32_t v = w + 1; v < W; ++v) c += __popcll(Rt[v] & Rs[v] & Rl[v]);
                k4 += c;
            }
        }
    }
}

// a split work item: te (10 bits) | s (10) | W - 1 (4) | run index j (8) -> ranks [8j, 8j+8)
__device__ __forceinline__ void dlr_split_item(const unsigned long long* __restrict__ R, unsigned long long rb, uint32_t pk,
                                               unsigned long long& k4) {
    const uint32_t te = pk & 0x3ffu, s = (pk >> 10) & 0x3ffu, W = ((pk >> 20) & 0xfu) + 1u, r0 = (pk >> 24) * kDlrRun;
    const unsigned long long* Rg = R + rb;
    if (W == 1) dlr_run<1>(Rg, te, s, 1, r0, k4);
    else if (W == 2) dlr_run<2>(Rg, te, s, 2, r0, k4);
    else if (W <= 4) dlr_run<4>(Rg, te, s, W, r0, k4);
    else dlr_run<0>(Rg, te, s, W, r0, k4);
}

// CUTS_DEBUG_TAIL_ALT (ablation): drain the 32 queued entries with one lane per
// triangle instead of one lane per entry — each entry's x (rows of <= 4 words) is staged in
// the warp's shared memory, a warp scan numbers the triangles, every round gives each lane
// one (binary search of the scan by shuffles) and the lane adds |x & {> l} & A_l|.
// Entries with wider rows keep the per-entry loop.
__device__ __forceinline__ void dlr_drain_tri(const unsigned long long* __restrict__ R, unsigned long long rb, uint32_t pk,
                                              bool own, unsigned long long* xs, unsigned long long& tri,
                                              unsigned long long& k4) {
    const int lane = threadIdx.x & 31;
    const uint32_t te = pk & 0x7ffu, s = (pk >> 11) & 0x7ffu, W = pk >> 22;
    const unsigned long long* Rg = R + rb;
    uint32_t n = 0;
    if (own && W > 4) dlr_tail_item(R, rb, pk, tri, k4);
    if (own && W <= 4) {
        const unsigned long long* Rt = Rg + (uint64_t)te * W;
        const unsigned long long* Rs = Rg + (uint64_t)s * W;
#pragma unroll
        for (int w = 0; w < 4; ++w) {
            const unsigned long long xw = (uint32_t)w < W ? (Rt[w] & Rs[w] & dlr_above(s, (uint32_t)w)) : 0ull;
            xs[lane * 4 + w] = xw;
            n += (uint32_t)__popcll(xw);
        }
        tri += n;
    }
    uint32_t incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
    }
    const uint32_t excl = incl - n;
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    __syncwarp();
    for (uint32_t j = 0; j < total; j += 32) {
        const uint32_t k = j + lane;
        uint32_t o = 0;
#pragma unroll
        for (uint32_t step = 16; step; step >>= 1) {
            const uint32_t v = __shfl_sync(0xffffffffu, incl, (int)(o + step - 1));
            if (v <= k) o += step;
        }
        uint32_t r = k - __shfl_sync(0xffffffffu, excl, (int)o);
        const unsigned long long orb = __shfl_sync(0xffffffffu, rb, (int)o);
        const uint32_t Wo = __shfl_sync(0xffffffffu, pk, (int)o) >> 22;
        if (k < total) {
            unsigned long long x[4];
#pragma unroll
            for (int w = 0; w < 4; ++w) x[w] = xs[o * 4 + w];
            uint32_t wl = 0;
#pragma unroll
            for (int w = 0; w < 4; ++w) {                   // the word holding the r-th member
                const uint32_t pc = (uint32_t)__popcll(x[w]);
                if (wl == (uint32_t)w && r >= pc) { r -= pc; wl = w + 1; }
            }
            unsigned long long xl = 0;
#pragma unroll
            for (int w = 0; w < 4; ++w) xl = (uint32_t)w == wl ? x[w] : xl;
            const uint32_t b = dlr_fns64(xl, r);
            const uint32_t l = 64u * wl + b;
            const unsigned long long* Rl = R + orb + (uint64_t)l * Wo;
            unsigned long long c = 0;
#pragma unroll
            for (int w = 0; w < 4; ++w) {
                const unsigned long long m = (uint32_t)w < wl ? 0ull
                                           : ((uint32_t)w == wl ? (b == 63u ? 0ull : (~0ull << (b + 1u))) : ~0ull);
                c += ((uint32_t)w < Wo && m) ? __popcll(x[w] & m & Rl[w]) : 0ull;
            }
            k4 += c;
        }
    }
    __syncwarp();
}

// Warps walk the written level-(b+1) chunk out[0, size) (children of level-b entries
// [e0, ..)) 32 entries at a time; each lane resolves its entry (e_t, G[s]) — parent
// from the trie, s = the rank-th member of A_t — and the entries with t < s go to a
// warp-private queue in shared memory, which is drained 32 at a time, so every lane of
// the bit-algebra loop holds work.  With count_bytes the §8.d model of both fused
// levels, computed per entry as the unshared pipeline would charge it (every
// level-(b+1) entry's extension and every level-(b+2) child's count-only extension).
template <bool count_bytes, int V>
__global__ void __launch_bounds__(256) k_dlr_tail(Graph g, Trie t, Dlr a, const uint64_t* __restrict__ cpos_b, uint64_t e0,
                                                  const uint2* __restrict__ out, uint64_t size,
                                                  unsigned long long* __restrict__ ctrl,
                                                  uint32_t lev1, uint32_t bw1, uint32_t bw2) {
    __shared__ unsigned long long q_rb[8][64];
    __shared__ uint32_t q_pk[8][64];
    __shared__ unsigned long long q_x[V == 1 ? 8 : 1][V == 1 ? 128 : 1];   // CUTS_DEBUG_TAIL_ALT: staged x words
    unsigned long long tri = 0, k4 = 0, b_plan = 0, b_ext = 0, b_out = 0, b_need = 0, b_ops = 0;
    const uint64_t c0 = cpos_b[e0];
    const int lane = threadIdx.x & 31, wq = threadIdx.x >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    uint32_t qn = 0;                                        // queued items (warp-uniform)
    for (uint64_t base = (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; base < size; base += nwarps * 32) {
        const uint64_t f = base + lane;
        bool up = false;
        unsigned long long rb = 0;
        uint32_t pk = 0;
        if (f < size) {
            const uint32_t e = out[f].y;
            const DlrGrp gr = dlr_group(a, e);
            const uint32_t te = (uint32_t)(e - gr.g0);
            const unsigned long long* Rt = a.R + gr.rb + (uint64_t)te * gr.W;
            const uint32_t s = dlr_select(Rt, gr.W, (uint32_t)(f - (cpos_b[e] - c0)));
            up = te < s;
            rb = gr.rb;
            pk = te | (s << 11) | (gr.W << 22);
            if (count_bytes) {
                // the unshared model: entry f extends to |A_t & A_s| children, each of which
                // counts |A_t & A_s & A_l| (same §8.d terms as the pipeline would charge)
                const unsigned long long* Rg = a.R + gr.rb;
                const unsigned long long* Rs = Rg + (uint64_t)s * gr.W;
                unsigned long long nx = 0, sx = 0, dl = 0;
                for (uint32_t w = 0; w < gr.W; ++w) {
                    const unsigned long long xw = Rt[w] & Rs[w];
                    nx += __popcll(xw);
                    for (unsigned long long y = xw; y; y &= y - 1) {
                        const uint32_t l = 64u * w + (uint32_t)(__ffsll((long long)y) - 1);
                        const unsigned long long* Rl = Rg + (uint64_t)l * gr.W;
                        for (uint32_t v = 0; v < gr.W; ++v) sx += __popcll(Rt[v] & Rs[v] & Rl[v]);
                        if ((bw2 >> lev1) & 1u) dl += __ldg(g.deg + a.lv[gr.g0 + l].x);
                    }
                }
                const unsigned long long d1 = bw_degree_sum(g, t, lev1, f, bw1);
                const unsigned long long d2 = bw_degree_sum(g, t, lev1, f, bw2 & ((1u << lev1) - 1u));
                b_plan += 8ull + 8ull * (lev1 - 1) + 16ull * __popc(bw1) + nx * (8ull + 8ull * lev1 + 16ull * __popc(bw2));
                b_ext += 4ull * d1 + 4ull * nx + 4ull * nx * d2 + 4ull * dl + 4ull * sx;
                b_out += 8ull * nx;
                b_need += 8ull + 16ull * gr.W + (up ? 8ull * nx * gr.W / 3 : 0ull);
                if (up) {     // word-ops of the symmetric bit algebra (the ALU roofline's unit)
                    unsigned long long ops = gr.W - (s >> 6);
                    for (uint32_t w = s >> 6; w < gr.W; ++w)
                        for (unsigned long long y = Rt[w] & Rs[w] & dlr_above(s, w); y; y &= y - 1) ops += gr.W - w;
                    b_ops += ops;
                }
            }
        }
        if (V == 2) {
            // split work items: an entry with |x| = n becomes ceil(n / kDlrRun) queue items
            uint32_t n = 0;
            if (up) {
                const uint32_t te = pk & 0x7ffu, s = (pk >> 11) & 0x7ffu, W = pk >> 22;
                const unsigned long long* Rt = a.R + rb + (uint64_t)te * W;
                const unsigned long long* Rs = a.R + rb + (uint64_t)s * W;
                for (uint32_t w = s >> 6; w < W; ++w) n += (uint32_t)__popcll(Rt[w] & Rs[w] & dlr_above(s, w));
                tri += n;
                pk = te | (s << 10) | ((W - 1) << 20);
            }
            const uint32_t nsub = (n + kDlrRun - 1) / kDlrRun;
            for (uint32_t j = 0;; ++j) {
                const bool want = j < nsub;
                const unsigned bj = __ballot_sync(0xffffffffu, want);
                if (!bj) break;
                if (want) {
                    const uint32_t pos = qn + __popc(bj & ((1u << lane) - 1u));
                    q_rb[wq][pos] = rb;
                    q_pk[wq][pos] = pk | (j << 24);
                }
                qn += __popc(bj);
                __syncwarp();
                if (qn >= 32) {
                    dlr_split_item(a.R, q_rb[wq][qn - 32 + lane], q_pk[wq][qn - 32 + lane], k4);
                    qn -= 32;
                    __syncwarp();
                }
            }
            continue;
        }
        const unsigned bal = __ballot_sync(0xffffffffu, up);
        if (up) {
            const uint32_t pos = qn + __popc(bal & ((1u << lane) - 1u));
            q_rb[wq][pos] = rb;
            q_pk[wq][pos] = pk;
        }
        qn += __popc(bal);
        __syncwarp();
        if (qn >= 32) {                                     // drain the 32 newest items
            if (V == 1) dlr_drain_tri(a.R, q_rb[wq][qn - 32 + lane], q_pk[wq][qn - 32 + lane], true, q_x[V == 1 ? wq : 0], tri, k4);
            else dlr_tail_item(a.R, q_rb[wq][qn - 32 + lane], q_pk[wq][qn - 32 + lane], tri, k4);
            qn -= 32;
            __syncwarp();
        }
    }
    if (V == 2) {
        if ((uint32_t)lane < qn) dlr_split_item(a.R, q_rb[wq][lane], q_pk[wq][lane], k4);
    } else if (V == 1) {
        if (qn) dlr_drain_tri(a.R, (uint32_t)lane < qn ? q_rb[wq][lane] : 0ull, (uint32_t)lane < qn ? q_pk[wq][lane] : 0u,
                              (uint32_t)lane < qn, q_x[V == 1 ? wq : 0], tri, k4);
    } else if ((uint32_t)lane < qn) {
        dlr_tail_item(a.R, q_rb[wq][lane], q_pk[wq][lane], tri, k4);
    }
    tri = warp_sum(tri) * 6ull;
    k4 = warp_sum(k4) * 24ull;
    if (lane == 0) {
        if (tri) atomicAdd(ctrl + kLrLevel, tri);
        add_u128(ctrl + kCountLo, k4);
    }
    if (count_bytes) {
        flush_model_bytes(b_plan, b_ext, b_out, b_need, ctrl);
        b_ops = warp_sum(b_ops);
        if (lane == 0 && b_ops) atomicAdd(ctrl + kTailOps, b_ops);
    }
}

// ---- the tail for wide groups (129..1024 members): a CTA per group, rows staged by TMA
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// Wide groups (129..1024 members, 3..16 row words) hold much of the tail's work and reuse
// their m x W row block across all their level-(b+1) entries: a CTA takes one such group
// at a time (dynamic queue over a CUB-selected list of their parent slots), one elected
// thread stages the block into shared memory with a single bulk copy (cp.async.bulk,
// completion on an mbarrier; blocks above kDlrSmemBytes stay in global memory), and the
// warps run the warp-queue algebra of k_dlr_tail over the group's stored entries with
// the rows read from shared memory.  Smaller groups go to k_dlr_tail_warp.
struct DlrWide {                      // a work list of parent slots (x = q - ea), ascending (CUB select)
    const uint32_t* __restrict__ x;
    uint32_t n;
};

__global__ void __launch_bounds__(256, 5) k_dlr_tail_cta(Dlr a, DlrOut L, uint64_t e1, const uint2* __restrict__ out,
                                                      unsigned long long* __restrict__ ctrl, DlrWide wide,
                                                      uint32_t xa, uint32_t xb) {
    const uint64_t e0 = L.e0;
    extern __shared__ __align__(16) unsigned long long srow[];
    __shared__ __align__(8) unsigned long long mbar;
    __shared__ uint32_t q_pk[8][64];
    __shared__ uint64_t s_q;
    unsigned long long tri = 0, k4 = 0;
    const int lane = threadIdx.x & 31, wq = threadIdx.x >> 5;
    const uint64_t cbase = a.cpos[a.ea];
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    uint32_t phase = 0;
    // the wide groups whose slots lie in [xa, xb] (the level-b entries of this chunk)
    uint32_t lo = 0, hi = wide.n;
    {
        uint32_t l = 0, h = wide.n;
        while (l < h) { const uint32_t mid = (l + h) / 2; if (wide.x[mid] < xa) l = mid + 1; else h = mid; }
        lo = l;
        h = wide.n;
        while (l < h) { const uint32_t mid = (l + h) / 2; if (wide.x[mid] <= xb) l = mid + 1; else h = mid; }
        hi = l;
    }
    for (;;) {
        if (threadIdx.x == 0) s_q = lo + atomicAdd(ctrl + kDlrWork, 1ull);
        __syncthreads();
        if (s_q >= hi) break;
        const uint64_t q = a.ea + wide.x[s_q];
        const uint64_t g0 = a.cpos[q] - cbase;
        const uint32_t m = (uint32_t)(a.cpos[q + 1] - a.cpos[q]);
        const uint32_t W = (m + 63) / 64;
        if (m <= 128 || m > (uint32_t)kDlrMaxM) { __syncthreads(); continue; }   // W <= 2: k_dlr_tail_warp
        const uint64_t t0 = g0 > e0 ? g0 : e0, t1 = (g0 + m < e1) ? g0 + m : e1;
        if (t0 >= t1) { __syncthreads(); continue; }
        const uint64_t F0 = dlr_child_off(L, t0, true), F1 = dlr_child_off(L, t1, true);
        const unsigned long long rb = a.roff[q - a.ea];
        const uint32_t bytes = (uint32_t)((((uint64_t)m * W + 1) & ~1ull) * 8);
        const bool staged = bytes <= kDlrSmemBytes;
        if (staged) {
            if (threadIdx.x == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // earlier generic reads of srow
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                             ::"r"(smem_u32(&mbar)), "r"(bytes) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(smem_u32(srow)), "l"(a.R + rb), "r"(bytes), "r"(smem_u32(&mbar)) : "memory");
            }
            uint32_t done = 0;
            while (!done) {
                asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                             : "=r"(done) : "r"(smem_u32(&mbar)), "r"(phase) : "memory");
            }
            phase ^= 1u;
        }
        const unsigned long long* Rg = staged ? srow : a.R + rb;
        uint32_t qn = 0;
        for (uint64_t base = F0 + (uint64_t)wq * 32; base < F1; base += 256) {
            const uint64_t f = base + lane;
            bool up = false;
            uint32_t pk = 0;
            if (f < F1) {
                const uint32_t e = out[f].y;
                const uint32_t te = (uint32_t)(e - g0);
                const uint32_t s = te < m ? dlr_select(Rg + (uint64_t)te * W, W, (uint32_t)(f - dlr_child_off(L, e, true)))
                                          : 0xffffffffu;
                if (s >= m) atomicAdd(ctrl + kErr, 1ull);          // cannot happen: the rows wrote this entry
                up = te < s && s < m;
                pk = te | (s << 11) | (W << 22);
            }
            const unsigned bal = __ballot_sync(0xffffffffu, up);
            if (up) {
                const uint32_t pos = qn + __popc(bal & ((1u << lane) - 1u));
                q_pk[wq][pos] = pk;
            }
            qn += __popc(bal);
            __syncwarp();
            if (qn >= 32) {
                const uint32_t pq = q_pk[wq][qn - 32 + lane];
                const uint32_t te = pq & 0x7ffu, s = (pq >> 11) & 0x7ffu;
                const unsigned long long* Rt = Rg + (uint64_t)te * W;
                const unsigned long long* Rs = Rg + (uint64_t)s * W;
                if (W == 2) dlr_tail_one<2>(Rt, Rs, Rg, 2, s, tri, k4);
                else if (W <= 4) dlr_tail_one<4>(Rt, Rs, Rg, W, s, tri, k4);
                else dlr_tail_one<0>(Rt, Rs, Rg, W, s, tri, k4);
                qn -= 32;
                __syncwarp();
            }
        }
        if ((uint32_t)lane < qn) {
            const uint32_t pq = q_pk[wq][lane];
            const uint32_t te = pq & 0x7ffu, s = (pq >> 11) & 0x7ffu;
            const unsigned long long* Rt = Rg + (uint64_t)te * W;
            const unsigned long long* Rs = Rg + (uint64_t)s * W;
            if (W == 2) dlr_tail_one<2>(Rt, Rs, Rg, 2, s, tri, k4);
            else if (W <= 4) dlr_tail_one<4>(Rt, Rs, Rg, W, s, tri, k4);
            else dlr_tail_one<0>(Rt, Rs, Rg, W, s, tri, k4);
        }
        __syncthreads();                                    // srow is free for the next group
    }
    tri = warp_sum(tri) * 6ull;
    k4 = warp_sum(k4) * 24ull;
    if (lane == 0) {
        if (tri) atomicAdd(ctrl + kLrLevel, tri);
        add_u128(ctrl + kCountLo, k4);
    }
}

// ---- the tail for narrow and mid groups: a warp per group --------------------------
// WM = 1: groups of 2..64 members (one row word; the narrow part of the split layout);
// WM = 2: 65..128 members (two words; in the wide part).  A warp claims a group, copies
// its m rows (<= 2 KB) into a warp-private slice of shared memory, then walks the
// group's stored level-(b+1) entries 32 at a time: lane per entry, s by a select on the
// staged row, the symmetric 4-clique algebra entirely on shared-memory rows.
template <int WM>
__global__ void __launch_bounds__(256) k_dlr_tail_warp(Dlr a, DlrOut L, uint64_t e1, const uint2* __restrict__ out,
                                                       unsigned long long* __restrict__ ctrl, DlrWide list,
                                                       uint32_t xa, uint32_t xb) {
    __shared__ unsigned long long srow[8][64 * WM * WM];
    unsigned long long tri = 0, k4 = 0;
    const int lane = threadIdx.x & 31, wq = threadIdx.x >> 5;
    const uint64_t e0 = L.e0, cbase = a.cpos[a.ea];
    uint32_t lo = 0, hi = list.n;
    {
        uint32_t l = 0, h = list.n;
        while (l < h) { const uint32_t mid = (l + h) / 2; if (list.x[mid] < xa) l = mid + 1; else h = mid; }
        lo = l;
        h = list.n;
        while (l < h) { const uint32_t mid = (l + h) / 2; if (list.x[mid] <= xb) l = mid + 1; else h = mid; }
        hi = l;
    }
    unsigned long long* rows = srow[wq];
    for (;;) {
        unsigned long long i = 0;
        if (lane == 0) i = lo + atomicAdd(ctrl + kDlrWork, (unsigned long long)(WM == 1 ? 8 : 2));
        i = __shfl_sync(0xffffffffu, i, 0);
        if (i >= hi) break;
        const unsigned long long iend = i + (WM == 1 ? 8 : 2) < hi ? i + (WM == 1 ? 8 : 2) : hi;
        for (; i < iend; ++i) {
            const uint64_t q = a.ea + list.x[i];
            const uint64_t g0 = a.cpos[q] - cbase;
            const uint32_t m = (uint32_t)(a.cpos[q + 1] - a.cpos[q]);
            const uint64_t t0 = g0 > e0 ? g0 : e0, t1 = (g0 + m < e1) ? g0 + m : e1;
            if (t0 >= t1) continue;                                      // warp-uniform
            const unsigned long long* R = a.R + a.roff[q - a.ea];
            for (uint32_t j = lane; j < 64u * WM * WM; j += 32) rows[j] = j < m * WM ? R[j] : 0ull;
            __syncwarp();
            const uint64_t F0 = dlr_child_off(L, t0, WM > 1), F1 = dlr_child_off(L, t1, WM > 1);
            for (uint64_t f = F0 + lane; f - lane < F1; f += 32) {
                if (f < F1) {
                    const uint32_t e = out[f].y;
                    const uint32_t te = (uint32_t)(e - g0);
                    const unsigned long long* Rt = rows + (uint64_t)(te & (64 * WM - 1)) * WM;
                    const uint32_t s = dlr_select(Rt, WM, (uint32_t)(f - dlr_child_off(L, e, WM > 1)));
                    if (te < s && s < 64u * WM) dlr_tail_one<WM>(Rt, rows + (uint64_t)s * WM, rows, WM, s, tri, k4);
                }
            }
            __syncwarp();
        }
    }
    tri = warp_sum(tri) * 6ull;
    k4 = warp_sum(k4) * 24ull;
    if (lane == 0) {
        if (tri) atomicAdd(ctrl + kLrLevel, tri);
        add_u128(ctrl + kCountLo, k4);
    }
}

// CUTS_DEBUG_GROUPS: log2 histogram of the children counts cnt[0..W) (the sizes of
// the next level's sibling groups): per bucket the groups, sum m, sum m^2
__global__ void k_group_hist(const uint64_t* __restrict__ cnt, uint32_t W, unsigned long long* __restrict__ h) {
    __shared__ unsigned long long s[48];
    if (threadIdx.x < 48) s[threadIdx.x] = 0;
    __syncthreads();
    for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < W; e += gridDim.x * blockDim.x) {
        const unsigned long long m = cnt[e];
        const int b = m ? min(15, 64 - __clzll((long long)m)) : 0;
        atomicAdd(&s[b * 3], 1ull);
        atomicAdd(&s[b * 3 + 1], m);
        atomicAdd(&s[b * 3 + 2], m * m);
    }
    __syncthreads();
    if (threadIdx.x < 48 && s[threadIdx.x]) atomicAdd(h + threadIdx.x, s[threadIdx.x]);
}

// ------------------------------------------------ SV intersection (ablation)
// Alg. 2 l.7-17, the scatter-vector intersection the paper rules
// out for GPUs because of its O(|V| x workers) space: here every warp owns a
// u8 scatter vector sv[|V|] in the arena (CUTS_DEBUG_SV; NEXT-2 ablation).
// Per entry the warp (1) scatters each backward list other than the source,
// sv[v]++ (coalesced reads, l.9-12), (2) collects: streams the source and keeps
// c iff sv[c] == number of those lists (l.14-16) — then the degree and
// injectivity filters and the warp-aggregated append as in k_extend — and (3)
// clears the lists' entries again.  Levels with one list (NL = 0) have nothing
// to intersect and use k_extend.  Count / write modes only.
template <int J, int NL, int M>
__global__ void __launch_bounds__(256) k_extend_sv(Graph g, QPlan q, uint64_t w0, uint32_t W,
                                                   const uint32_t* __restrict__ path_s,
                                                   const uint64_t* __restrict__ src_off,
                                                   const uint64_t* __restrict__ offs,
                                                   const uint64_t* __restrict__ lst_off,
                                                   const uint32_t* __restrict__ lst_len,
                                                   uint64_t t0, uint64_t t1, uint2* __restrict__ out_level,
                                                   uint64_t cap, unsigned long long* __restrict__ ctrl,
                                                   uint8_t* __restrict__ sv_base, uint64_t sv_stride) {
    static_assert(NL >= 1, "SV needs a list to intersect");
    __shared__ uint32_t s_ent[2];
    if (threadIdx.x == 0) {
        uint64_t tt[2] = {t0, t1 - 1};
        for (int z = 0; z < 2; ++z) {
            uint32_t lo = 0, hi = W - 1;
            while (lo < hi) {
                uint32_t mid = (lo + hi + 1) >> 1;
                if (offs[mid] <= tt[z]) lo = mid; else hi = mid - 1;
            }
            s_ent[z] = lo;
        }
    }
    __syncthreads();
    const uint32_t ea = s_ent[0];
    const uint32_t nent = s_ent[1] - ea + 1;
    const int lane = threadIdx.x & 31;
    const uint64_t gwarp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    uint8_t* __restrict__ sv = sv_base + gwarp * sv_stride;
    const uint32_t qd = q.qdeg[J];
    const uint32_t qmin = 1u;                     // undirected: list members have deg >= 1
    unsigned long long my_count = 0;
    unsigned int* work = (unsigned int*)(ctrl + kWork);
    for (;;) {
        uint32_t ei = 0;
        if (lane == 0) ei = atomicAdd(work, 1u);
        ei = __shfl_sync(0xffffffffu, ei, 0);
        if (ei >= nent) break;
        const uint32_t e = ea + ei;
        const uint64_t o0 = offs[e], o1 = offs[e + 1];
        const uint32_t ilo = (uint32_t)((o0 > t0 ? o0 : t0) - o0);
        const uint32_t ihi = (uint32_t)((o1 < t1 ? o1 : t1) - o0);
        const uint64_t so = src_off[e];
        uint32_t path[J];
#pragma unroll
        for (int p = 0; p < J; ++p) path[p] = path_s[(size_t)p * W + e];
        uint64_t lo_[NL];
        uint32_t ln_[NL];
        uint32_t nlists = 0;
#pragma unroll
        for (int x = 0; x < NL; ++x) {
            lo_[x] = lst_off[(size_t)x * W + e];
            ln_[x] = lst_len[(size_t)x * W + e];
            nlists += ln_[x] != kSkip ? 1u : 0u;
        }
        // (1) scatter: sv[v]++ for every v of every other list (distinct within a list)
#pragma unroll
        for (int x = 0; x < NL; ++x) {
            if (ln_[x] == kSkip) continue;
            const uint32_t* l = g.col + lo_[x];
            for (uint32_t i = lane; i < ln_[x]; i += 32) sv[__ldg(l + i)] += 1;
            __syncwarp();
        }
        // (2) collect over the source items of this chunk
        const bool pk = g.colx != nullptr && qd > qmin;
        const uint32_t* __restrict__ src = (pk ? g.colx : g.col) + so;
        const uint32_t umask = pk ? kPackMask : 0xffffffffu;
        for (uint32_t b = ilo; b < ihi; b += 32) {
            const uint32_t i = b + lane;
            const bool act = i < ihi;
            const uint32_t raw = act ? __ldg(src + i) : 0u;
            const uint32_t c = raw & umask;
            bool ok = act && sv[c] == nlists;
#pragma unroll
            for (int p = 0; p < J; ++p) ok = ok && path[p] != c;
            if (qd > qmin) ok = ok && (pk ? (raw >> kPackShift) : __ldg(g.deg + c)) >= qd;
            if (M == kCount) {
                my_count += ok ? 1 : 0;
            } else {
                const unsigned m = __ballot_sync(0xffffffffu, ok);
                unsigned long long pos0 = 0;
                if (lane == 0 && m) pos0 = atomicAdd(ctrl + kCursor, (unsigned long long)__popc(m));
                pos0 = __shfl_sync(0xffffffffu, pos0, 0);
                const unsigned long long pos = pos0 + __popc(m & ((1u << lane) - 1u));
                if (ok && pos < cap) out_level[pos] = make_uint2(c, (uint32_t)(w0 + e));
            }
        }
        __syncwarp();
        // (3) clear what (1) set
#pragma unroll
        for (int x = 0; x < NL; ++x) {
            if (ln_[x] == kSkip) continue;
            const uint32_t* l = g.col + lo_[x];
            for (uint32_t i = lane; i < ln_[x]; i += 32) sv[__ldg(l + i)] = 0;
        }
        __syncwarp();
    }
    if (M == kCount) {
        my_count = warp_sum(my_count);
        if (lane == 0) add_u128(ctrl + kCountLo, my_count);
    }
}

// ------------------------------------------------- ordered-level chunking
// Largest eb in [ea, W] with cpos[eb] - cpos[ea] <= cap (children of entries
// [ea, eb) fit the level chunk).  out: eb, children, items [offs[ea], offs[eb]),
// and for a single oversized entry its item end offs[ea+1].
__global__ void k_find_chunk(const uint64_t* __restrict__ cpos, const uint64_t* __restrict__ offs, uint32_t W,
                             uint32_t ea, uint64_t cap, unsigned long long* __restrict__ out) {
    const uint64_t c0 = cpos[ea];
    uint32_t lo = ea, hi = W;            // invariant: cpos[lo] - c0 <= cap
    while (lo < hi) {
        const uint32_t mid = lo + (hi - lo + 1) / 2;
        if (cpos[mid] - c0 <= cap) lo = mid; else hi = mid - 1;
    }
    out[0] = lo;
    out[1] = cpos[lo] - c0;
    out[2] = offs[ea];
    out[3] = offs[lo];
    out[4] = offs[ea + 1 <= W ? ea + 1 : W];
}

// ------------------------------------------------- binned virtual warps
// The paper's first strategy ("group the paths based on the work
// into bins and use virtual warps to process the bins"; kept as the NEXT-2
// ablation CUTS_DEBUG_BINNED): entry e goes to the bin of the smallest virtual
// warp G in {8, 16, 32} with ub(e) <= G (ub > 16: the 32-lane bin); entries
// with no candidates are dropped.  bins[b * W + i] = i-th entry of bin b,
// cnt[b] = bin size.
__global__ void k_bin(const uint64_t* __restrict__ ub, uint32_t W, uint32_t* __restrict__ bins,
                      unsigned long long* __restrict__ cnt) {
    for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < W; e += gridDim.x * blockDim.x) {
        const uint64_t u = ub[e];
        if (u == 0) continue;
        const int b = u <= 8 ? 0 : (u <= 16 ? 1 : 2);
        const unsigned long long i = atomicAdd(cnt + b, 1ull);
        bins[(size_t)b * W + i] = e;
    }
}

// ---------------------------------------------------------- work donation
// Flat prefixes (reading P24): a donated unit of work is a J-vertex partial
// embedding in matching-order positions, rows of J u32.  Export walks the trie
// of the donor (the path recovery of P:956-958); import rebuilds a chain trie
// (level l entry i = (row[i][l-1], parent i)) that the receiver extends from
// level J on, so no trie is shipped (cf. the extraction cost named at P:1168-1176).
template <int J>
__global__ void k_prefix_export(Trie t, uint64_t e0, uint64_t cnt, uint32_t* __restrict__ rows) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint2 cur = t.lv[J][e0 + i];
        uint32_t* row = rows + i * J;
        row[J - 1] = cur.x;
        uint32_t idx = cur.y;
#pragma unroll
        for (int p = J - 2; p >= 0; --p) {
            cur = t.lv[p + 1][idx];
            row[p] = cur.x;
            idx = cur.y;
        }
    }
}

// lv[l] (l = 1..J) each hold cnt entries: (rows[i][l-1], i)
// multi-GPU partition below level 1 (cuts_set_partition_depth): positions p0, p0 +
// nparts, ... of the seeded shuffle of the whole level-J list, each exported as a flat
// row of J vertices in matching-order positions (the seed format of cuts_set_prefixes)
template <int J>
__global__ void k_prefix_slice(Trie t, Shuffle sh, uint64_t p0, uint32_t nparts, uint64_t cnt,
                               uint32_t* __restrict__ rows) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint2 cur = t.lv[J][sh.apply(p0 + i * nparts)];
        uint32_t* row = rows + i * J;
        row[J - 1] = cur.x;
        uint32_t idx = cur.y;
#pragma unroll
        for (int p = J - 2; p >= 0; --p) {
            cur = t.lv[p + 1][idx];
            row[p] = cur.x;
            idx = cur.y;
        }
    }
}

__global__ void k_prefix_import(const uint32_t* __restrict__ rows, uint32_t J, uint64_t cnt, Trie t) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt;
         i += (uint64_t)gridDim.x * blockDim.x) {
        for (uint32_t l = 1; l <= J; ++l)
            const_cast<uint2*>(t.lv[l])[i] = make_uint2(rows[i * J + l - 1], (uint32_t)i);
    }
}

// ---------------------------------------------------------------- trie decode
struct DecodeArgs {
    const uint32_t* ca[kMaxK];
    const uint32_t* pa[kMaxK];
    uint64_t size[kMaxK];
    uint32_t L;
};

__global__ void k_trie_decode(DecodeArgs a, uint32_t* __restrict__ out, unsigned long long* ctrl) {
    const uint64_t n = a.size[a.L - 1];
    for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t at = x;
        for (int l = (int)a.L - 1; l >= 0; --l) {
            if (at >= a.size[l]) { atomicExch(ctrl + kErr, 1ull); break; }
            out[x * a.L + l] = a.ca[l][at];
            if (l > 0) at = a.pa[l][at];
        }
    }
}

}  // namespace cuts
