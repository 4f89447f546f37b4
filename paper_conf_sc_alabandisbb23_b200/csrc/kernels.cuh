// kernels.cuh -- sm_100a kernels of the ECL-SCC hot path.
//
// Citation key: P:n = PAPER.md line n.  Steps:
//   a1    k_validate, k_indeg, k_csc_scatter    CSR -> CSC transpose of the input
//   a2/a7 k_keep_count, k_compact_count,        Phase 3 edge removal
//         k_compact_map, k_compact_scatter      fused with one Trim-1 round and the
//                                               compaction of CSR and CSC
//   a3    (inside k_compact_map)                Phase 1 of the next iteration
//   a4-a6 k_prop_tile, k_prop_heavy             Phase 2 max propagation with
//                                               block-local fixed points
//   a8    (inside k_compact_map)                final labels
//
// Layout: after every compaction the working graph is renumbered
// to LOCAL indices 0..na-1 (stable, so local order = vertex-ID order).  act[i] is the
// vertex ID of local i, cin[i]/cout[i] its signatures (values are vertex IDs), and
// optr/oadj (out-edges, CSR) and iptr/iadj (in-edges, CSC) hold local indices.  Later
// iterations therefore touch small, dense arrays.
#pragma once
#include "common.cuh"

namespace eclscc {

constexpr int TILE = 2048;          // vertices per block-local fixed point
constexpr int TILE_THREADS = 512;   // threads per tile CTA
constexpr int VPT = TILE / TILE_THREADS;
constexpr int HEAVY_T = 64;         // rows longer than this are reduced by k_prop_heavy
constexpr int CHUNK = 512;          // edges per heavy-row chunk (one warp)

// Heavy-row chunk (a piece of one long adjacency row, one warp each)
struct Chunk {
    int32_t i;      // local vertex
    int32_t dir;    // 0: out-row (pull cout), 1: in-row (pull cin)
    int32_t beg, end;
    int32_t first;  // index of the first chunk of the same row (rows are contiguous runs)
};

// ------------------------------------------------------------------ init / validation
static __global__ void k_validate(int32_t n, int64_t nnz, const int32_t* __restrict__ rp,
                           const int32_t* __restrict__ ci, int* __restrict__ err) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int bad = 0;
    for (int64_t v = t0; v < n; v += stride) {
        const int32_t a = rp[v], b = rp[v + 1];
        if (a > b) bad = 1;
        if (v == 0 && a != 0) bad = 1;
        if (v == n - 1 && (int64_t)b != nnz) bad = 1;
    }
    for (int64_t e = t0; e < nnz; e += stride) {
        const int32_t c = ci[e];
        if (c < 0 || c >= n) bad = 1;
    }
    if (bad) *err = 1;
}

// ------------------------------------------------------------------ a1: CSR -> CSC
// in-degree histogram and (RANK) per edge its rank among the in-edges of its destination:
// edge-parallel returning atomics (no per-row serial chain), four independent per thread.
// Without RANK (power-law inputs: returning atomics on hub destinations serialise) the
// histogram uses fire-and-forget reductions and the scatter takes cursor atomics.
template <bool RANK>
static __global__ void __launch_bounds__(256) k_indeg_rank(int64_t nnz, const int32_t* __restrict__ ci,
                                                           int32_t* __restrict__ ideg, int32_t* __restrict__ rank) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t e0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e0 < nnz; e0 += 4 * stride) {
        int w[4], r[4];
#pragma unroll
        for (int q = 0; q < 4; q++) w[q] = e0 + q * stride < nnz ? __ldg(ci + e0 + q * stride) : -1;
#pragma unroll
        for (int q = 0; q < 4; q++) {
            if (!RANK && w[q] >= 0) atomicAdd(&ideg[w[q]], 1);
            r[q] = RANK && w[q] >= 0 ? atomicAdd(&ideg[w[q]], 1) : 0;
        }
        if (RANK)
#pragma unroll
            for (int q = 0; q < 4; q++)
                if (w[q] >= 0) rank[e0 + q * stride] = r[q];
    }
}

// one thread per source row: edge k = u -> w lands at iadj[iptr[w] + rank[k]] (RANK) or at
// a cursor slot; rows longer than HEAVY are spread over the warp, rows longer than HEAVY_T
// go to k_csc_scatter_chunks
template <bool RANK>
__device__ __forceinline__ int csc_slot(const int32_t* __restrict__ rank, int32_t* cursor, int k, int w) {
    return RANK ? __ldg(rank + k) : atomicAdd(cursor + w, 1);
}
template <bool RANK>
static __global__ void __launch_bounds__(256) k_csc_scatter(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                              const int32_t* __restrict__ iptr, const int32_t* __restrict__ rank, int32_t* cursor,
                              int32_t* __restrict__ iadj, unsigned long long* __restrict__ local_e) {
    const int lane = threadIdx.x & 31;
    const int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool valid = u < n;
    int b = 0, e = 0;
    if (valid) { b = __ldg(rp + u); e = __ldg(rp + u + 1); }
    if (e - b > HEAVY_T) e = b;                          // long row: k_csc_scatter_chunks
    unsigned nloc = 0;                                   // storage locality of the numbering
    if (valid && e - b <= HEAVY)
        for (int k = b; k < e; k += 4) {                 // loads of a batch issued before use
            int w[4], r[4], o[4];
#pragma unroll
            for (int q = 0; q < 4; q++) {
                w[q] = k + q < e ? __ldg(ci + k + q) : 0;
                r[q] = RANK && k + q < e ? __ldg(rank + k + q) : 0;
            }
#pragma unroll
            for (int q = 0; q < 4; q++) o[q] = __ldg(iptr + w[q]);
#pragma unroll
            for (int q = 0; q < 4; q++)
                if (k + q < e) {
                    nloc += ((w[q] ^ (int)u) >> 11) == 0;
                    iadj[o[q] + (RANK ? r[q] : atomicAdd(cursor + w[q], 1))] = (int32_t)u;
                }
        }
    {   // one atomic per block on the single counter (one per warp serialised ~0.5M in L2)
        __shared__ unsigned s_loc[256 / WARP];
        nloc = __reduce_add_sync(FULL, nloc);
        if (lane == 0) s_loc[threadIdx.x >> 5] = nloc;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned t = 0;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += s_loc[w];
            if (t) atomicAdd(local_e, (unsigned long long)t);
        }
    }
    unsigned hm = __ballot_sync(FULL, valid && e - b > HEAVY);
    while (hm) {
        const int src = __ffs(hm) - 1;
        hm &= hm - 1;
        const int sb = __shfl_sync(FULL, b, src), se = __shfl_sync(FULL, e, src);
        const int su = __shfl_sync(FULL, (int)u, src);
        for (int k = sb + lane; k < se; k += WARP) {
            const int w = __ldg(ci + k);
            iadj[__ldg(iptr + w) + csc_slot<RANK>(rank, cursor, k, w)] = su;
        }
    }
}

// ------------------------------------------------------------------ Phase 3 predicates
// keep(i->k) in iteration >= 2 (P:147 negated): both endpoints carry the same
// (in, out) pair and that pair is unfinished (in != out; checked once per row via `live`).
// Evaluated from either end: the row owner's pair (a, b) is passed in, the other
// endpoint's pair is gathered.  In the first removal (FIRST) every edge except a
// self-loop is kept (DESIGN reading 9).
// With the 4-signature variant (mi != nullptr) the minimum pair (c, d) must agree as well.
template <bool FIRST, bool FOUR = false>
__device__ __forceinline__ bool keep_edge(int owner, int a, int b, int other, const int32_t* __restrict__ cin,
                                          const int32_t* __restrict__ cout, const int2* __restrict__ s2 = nullptr,
                                          int c = 0, int d = 0, const int32_t* __restrict__ mi = nullptr,
                                          const int32_t* __restrict__ mo = nullptr) {
    if (FIRST) return other != owner;
    bool k;
    if (s2) {                                            // interleaved copy: one 8-byte gather
        const int2 x = __ldg(s2 + other);
        k = (x.x == a) & (x.y == b);
    } else {
        // both loads are issued unconditionally (no short circuit): callers batch these gathers
        k = (__ldg(cin + other) == a) & (__ldg(cout + other) == b);
    }
    if (FOUR) k &= (__ldg(mi + other) == c) & (__ldg(mo + other) == d);
    return k;
}
// Phase 3 of power-law graphs: the signatures interleaved for one gather per far end
static __global__ void k_pack_sig(int32_t na, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                  int2* __restrict__ sig2) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < na; v += (int64_t)gridDim.x * blockDim.x)
        sig2[v] = make_int2(__ldg(cin + v), __ldg(cout + v));
}
// Trim-1 on the kept graph: no kept in-edge or no kept out-edge
// kept degrees are interleaved (kio[x] = {in, out}): one 8-byte gather per far end
__device__ __forceinline__ bool trimmed(const int2* __restrict__ kio, int x) {
    const int2 k = __ldg(kio + x);
    return (k.x == 0) | (k.y == 0);
}
// Small-degree graphs (every row <= KW_DEG entries per direction: meshes), one 4-byte keep word
// per vertex instead of kio (8 B) + emask (8 B): byte 0 kept in-degree, byte 1 kept out-degree,
// byte 2 the out-row mask, byte 3 the in-row mask (Phase 3's kept entries; after the trim, the
// survivors -- the degree bytes, which other threads' trim tests read, stay as they were)
constexpr int KW_DEG = 8;
static_assert(KW_DEG * 32 < 1024, "k_compact_map packs the warp prefixes of the survivor degrees in 10 bits");
__device__ __forceinline__ bool trimmed_kw(const uint32_t* __restrict__ kw, int x) {
    const uint32_t w = __ldg(kw + x);
    return ((w & 0xFFu) == 0) | ((w & 0xFF00u) == 0);
}

struct RowCtx {
    int ob, oe, ib, ie, a, b, c, d;       // (c, d): the minimum pair (4-signature variant)
    bool valid, live;
};

template <bool FIRST, bool FOUR = false>
__device__ __forceinline__ RowCtx load_row(const WGraph& g, int64_t i, const int32_t* __restrict__ cin,
                                           const int32_t* __restrict__ cout) {
    RowCtx r{};
    r.valid = i < g.na;
    if (r.valid) {
        r.ob = g.optr[i]; r.oe = g.optr[i + 1];
        r.ib = g.iptr[i]; r.ie = g.iptr[i + 1];
        if (!FIRST) { r.a = cin[i]; r.b = cout[i]; }
        if (!FIRST && FOUR) { r.c = g.min_in[i]; r.d = g.min_out[i]; }
    }
    r.live = r.valid && (FIRST || r.a != r.b);
    return r;
}

// count edges of one row (light: by the lane, heavy: by the whole warp) that satisfy P
template <typename P>
__device__ __forceinline__ int count_row(const int32_t* __restrict__ adj, int rb, int re, bool go, int lane, P pred,
                                         bool chunked = false, bool light = true) {
    int c = 0;
    if (chunked && re - rb > HEAVY_T) go = false;      // long row: the chunk kernels count it
    if (light && go && re - rb <= HEAVY)
        for (int e = rb; e < re; e++) c += pred(__ldg(adj + e));
    unsigned hm = __ballot_sync(FULL, go && re - rb > HEAVY);
    while (hm) {
        const int src = __ffs(hm) - 1;
        hm &= hm - 1;
        const int sb = __shfl_sync(FULL, rb, src), se = __shfl_sync(FULL, re, src);
        const P bp = pred.bcast(src);
        int cc = 0;
        for (int e = sb + lane; e < se; e += WARP) cc += bp(__ldg(adj + e));
        cc = warp_sum(cc);
        if (lane == src) c = cc;
    }
    return c;
}

// predicate objects: evaluated for the row owner's lane; bcast(src) gives lane src's
// predicate to the whole warp (all lanes must call it)
template <bool FIRST, bool FOUR = false>
struct KeepPred {
    int i, a, b;
    const int32_t *cin, *cout;
    const int2* s2;
    int c, d;
    const int32_t *mi, *mo;
    __device__ __forceinline__ bool operator()(int k) const { return keep_edge<FIRST, FOUR>(i, a, b, k, cin, cout, s2, c, d, mi, mo); }
    __device__ __forceinline__ KeepPred bcast(int src) const {
        KeepPred p = *this;
        p.i = __shfl_sync(FULL, i, src); p.a = __shfl_sync(FULL, a, src); p.b = __shfl_sync(FULL, b, src);
        p.c = __shfl_sync(FULL, c, src); p.d = __shfl_sync(FULL, d, src);
        return p;
    }
};
template <bool FIRST, bool TRIM, bool FOUR = false>
struct SurvivePred {
    int i, a, b;
    const int32_t *cin, *cout;
    const int2* kio;
    const int2* s2;
    int c, d;
    const int32_t *mi, *mo;
    __device__ __forceinline__ bool operator()(int k) const {
        return keep_edge<FIRST, FOUR>(i, a, b, k, cin, cout, s2, c, d, mi, mo) & !(TRIM && trimmed(kio, k));
    }
    __device__ __forceinline__ SurvivePred bcast(int src) const {
        SurvivePred p = *this;
        p.i = __shfl_sync(FULL, i, src); p.a = __shfl_sync(FULL, a, src); p.b = __shfl_sync(FULL, b, src);
        p.c = __shfl_sync(FULL, c, src); p.d = __shfl_sync(FULL, d, src);
        return p;
    }
};

// Light rows as bit masks (bit k = entry k of the row satisfies the predicate).  Phase 3
// evaluates keep() once, in k_keep_count; k_compact_count then gathers only the trim
// degrees of the kept entries and k_compact_scatter only the new indices of the
// survivors (the predicates used to be re-evaluated, with their gathers, in all three).
template <typename P>
__device__ __forceinline__ void mask_light2(const int32_t* __restrict__ oadj, int ob, int no,
                                            const int32_t* __restrict__ iadj, int ib, int ni, int self, P pred,
                                            unsigned& mo, unsigned& mi) {
    for (int k = 0; k < no || k < ni; k += 4) {
        int xo[4], xi[4];
#pragma unroll
        for (int q = 0; q < 4; q++) {
            xo[q] = k + q < no ? __ldg(oadj + ob + k + q) : self;
            xi[q] = k + q < ni ? __ldg(iadj + ib + k + q) : self;
        }
#pragma unroll
        for (int q = 0; q < 4; q++) {
            mo |= (unsigned)((int)pred(xo[q]) & (int)(k + q < no)) << (k + q);
            mi |= (unsigned)((int)pred(xi[q]) & (int)(k + q < ni)) << (k + q);
        }
    }
}
// keep the set bits of m whose entry's far end is not trimmed (batches of 4 entries)
template <bool KW = false>
__device__ __forceinline__ unsigned trim_mask(const int32_t* __restrict__ adj, int b, unsigned m, int self,
                                              const int2* __restrict__ kio, const uint32_t* __restrict__ kw = nullptr) {
    unsigned out = 0;
    while (m) {
        int k[4], x[4];
#pragma unroll
        for (int q = 0; q < 4; q++) {
            k[q] = m ? __ffs(m) - 1 : -1;
            m &= m - 1;
        }
#pragma unroll
        for (int q = 0; q < 4; q++) x[q] = k[q] >= 0 ? __ldg(adj + b + k[q]) : self;
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (k[q] >= 0 && !(KW ? trimmed_kw(kw, x[q]) : trimmed(kio, x[q]))) out |= 1u << k[q];
    }
    return out;
}
// write the entries of m (in row order) as new local indices from dst[pos]
__device__ __forceinline__ void emit_mask(const int32_t* __restrict__ adj, int b, unsigned m, int self,
                                          const int32_t* __restrict__ newidx, int32_t* __restrict__ dst, int pos) {
    while (m) {
        int k[4], y[4];
#pragma unroll
        for (int q = 0; q < 4; q++) {
            k[q] = m ? __ffs(m) - 1 : -1;
            m &= m - 1;
        }
#pragma unroll
        for (int q = 0; q < 4; q++) y[q] = __ldg(newidx + (k[q] >= 0 ? __ldg(adj + b + k[q]) : self));
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (k[q] >= 0) dst[pos++] = y[q];
    }
}

// Tile-pack output of the compaction scatter (pack.cuh layout).  When pnin is set, the
// scatter also writes each survivor's slot words and appends its cut edges to its tile's
// list, so Phase 2 needs no separate k_tile_pack pass over the new graph; a row longer
// than HEAVY (warp path, no masks) sets *bad and the driver falls back to k_tile_pack.
struct PackOut {
    unsigned long long* pnin;
    unsigned long long* pnout;
    int2* ext;
    int* ext_cnt;
    int* bad;
};
constexpr unsigned long long PK_EMPTY = 0x0800080008000800ull;   // four empty slots (pack.cuh PSLOTS_EMPTY)
constexpr int PK_DIR = 0x8000;                                  // out-edge mark (pack.cuh EXT_DIR)
constexpr unsigned long long PK_SLOW = 0x8000ull << 48;         // > 4 intra-tile neighbours (SLOW_MARK)

__device__ __forceinline__ void pk_add(unsigned long long& pk, int& ns, unsigned idx) {
    pk &= ~(0xFFFFull << (16 * ns));
    pk |= (unsigned long long)idx << (16 * ns);
    ns++;
}
// emit_mask plus the pack of local vertex j (tile base tb): survivors in j's tile fill the
// slot word (returned); the others are counted in nc (they become cut edges of the tile,
// written by emit_cut once the warp has reserved their slots)
__device__ __forceinline__ unsigned long long emit_mask_pack(const int32_t* __restrict__ adj, int b, unsigned m, int self,
                                                             const int32_t* __restrict__ newidx, int32_t* __restrict__ dst,
                                                             int pos, int tb, int& nc) {
    unsigned long long pk = PK_EMPTY;
    int ns = 0;
    while (m) {
        int k[4], y[4];
#pragma unroll
        for (int q = 0; q < 4; q++) {
            k[q] = m ? __ffs(m) - 1 : -1;
            m &= m - 1;
        }
#pragma unroll
        for (int q = 0; q < 4; q++) y[q] = __ldg(newidx + (k[q] >= 0 ? __ldg(adj + b + k[q]) : self));
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (k[q] >= 0) {
                dst[pos++] = y[q];
                if ((unsigned)(y[q] - tb) < (unsigned)TILE) {
                    if (ns < 4) pk_add(pk, ns, (unsigned)(y[q] - tb));
                    else pk |= PK_SLOW;
                } else {
                    nc++;
                }
            }
    }
    return pk;
}
// the cut edges of one row (the survivors of m outside tile tb) as {far end, (j - tb) | dir}
__device__ __forceinline__ void emit_cut(const int32_t* __restrict__ adj, int b, unsigned m,
                                         const int32_t* __restrict__ newidx, int j, int tb, int dir,
                                         int2* __restrict__ E, int& at) {
    while (m) {
        const int k = __ffs(m) - 1;
        m &= m - 1;
        const int y = __ldg(newidx + __ldg(adj + b + k));
        if ((unsigned)(y - tb) >= (unsigned)TILE) E[at++] = make_int2(y, (j - tb) | dir);
    }
}

// kept in/out degree per local vertex (light rows: also the kept entries as bit masks)
constexpr int TPB_COMPACT = 256;     // block size of the compaction kernels (driver TPB)
template <bool FIRST, bool FOUR, bool KW = false>
static __global__ void __launch_bounds__(TPB_COMPACT) k_keep_count(WGraph g, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                             int2* __restrict__ kio, int chunked, int2* __restrict__ hcnt,
                             uint2* __restrict__ emask) {
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const RowCtx r = load_row<FIRST, FOUR>(g, i, cin, cout);
    KeepPred<FIRST, FOUR> pred{(int)i, r.a, r.b, cin, cout, g.sig2, r.c, r.d, g.min_in, g.min_out};
    unsigned mo = 0, mi = 0;
    mask_light2(g.oadj, r.ob, r.live && r.oe - r.ob <= HEAVY ? r.oe - r.ob : 0, g.iadj, r.ib,
                r.live && r.ie - r.ib <= HEAVY ? r.ie - r.ib : 0, (int)(r.valid ? i : 0), pred, mo, mi);
    int co = __popc(mo), ci = __popc(mi);
    if (KW) {                                        // (no row is longer than KW_DEG)
        if (r.valid) ((uint32_t*)emask)[i] = (uint32_t)ci | (uint32_t)co << 8 | mo << 16 | mi << 24;
        return;
    }
    co += count_row(g.oadj, r.ob, r.oe, r.live, lane, pred, chunked, false);
    ci += count_row(g.iadj, r.ib, r.ie, r.live, lane, pred, chunked, false);
    if (r.valid) {
        kio[i] = make_int2(ci, co);
        emask[i] = make_uint2(mo, mi);
        if (chunked) hcnt[i] = make_int2(0, 0);
    }
    // the number of kept edges is the sum of the kept out-degrees: k_compact_count carries it
    // through the compaction scan (lane .w), so no kernel counts it on a single address
}

// per-vertex surviving (kept, not trimmed) degrees and per-warp totals (alive, out, in, kept)
template <bool FIRST, bool TRIM, bool FOUR, bool KW = false>
static __global__ void k_compact_count(WGraph g, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                const int2* __restrict__ kio,
                                int2* __restrict__ cnt, int4* __restrict__ wsum, int chunked,
                                const int2* __restrict__ hcnt, uint2* __restrict__ emask) {
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const RowCtx r = load_row<FIRST, FOUR>(g, i, cin, cout);
    int nout = 0, nin = 0, kept = 0;
    if (KW) {                                          // small degrees: the 4-byte keep words
        uint32_t* kw = (uint32_t*)emask;
        if (r.valid) {
            const uint32_t w = kw[i];
            kept = (int)((w >> 8) & 0xFFu);
            const bool go = r.live && ((w & 0xFFu) != 0) && ((w & 0xFF00u) != 0);
            unsigned so = (w >> 16) & 0xFFu, si = w >> 24;
            if (TRIM) {
                so = go ? trim_mask<true>(g.oadj, r.ob, so, (int)i, nullptr, kw) : 0u;
                si = go ? trim_mask<true>(g.iadj, r.ib, si, (int)i, nullptr, kw) : 0u;
                kw[i] = (w & 0xFFFFu) | so << 16 | si << 24;
            } else if (!r.live) {
                so = si = 0;
            }
            nout = __popc(so);
            nin = __popc(si);                          // (k_compact_map counts them from the word)
        }
        const int alive = (nout + nin) > 0;
        const int sa = warp_sum(alive), so_ = warp_sum(nout), si_ = warp_sum(nin), sk = warp_sum(kept);
        if (lane == 0) wsum[i >> 5] = make_int4(sa, so_, si_, sk);
        return;
    }
    if (!TRIM) {
        if (r.live) { const int2 k = kio[i]; nout = k.y; nin = k.x; }   // survivors = kept: the masks stand
    } else {
        const bool go = r.live && !trimmed(kio, (int)i);
        SurvivePred<FIRST, TRIM, FOUR> pred{(int)i, r.a, r.b, cin, cout, kio, g.sig2, r.c, r.d, g.min_in, g.min_out};
        if (r.valid) {                                   // light rows: the kept entries' far ends
            const uint2 km = emask[i];
            const unsigned so = go && r.oe - r.ob <= HEAVY ? trim_mask(g.oadj, r.ob, km.x, (int)i, kio) : 0u;
            const unsigned si = go && r.ie - r.ib <= HEAVY ? trim_mask(g.iadj, r.ib, km.y, (int)i, kio) : 0u;
            emask[i] = make_uint2(so, si);
            nout = __popc(so);
            nin = __popc(si);
        }
        nout += count_row(g.oadj, r.ob, r.oe, go, lane, pred, chunked, false);
        nin += count_row(g.iadj, r.ib, r.ie, go, lane, pred, chunked, false);
        if (chunked && r.valid) {                       // long rows: counted by k_count_chunks
            const int2 h = hcnt[i];
            nout += h.x;
            nin += h.y;
        }
    }
    if (r.valid) cnt[i] = make_int2(nout, nin);
    int alive = (nout + nin) > 0;
    // partitioned mode: an unfinished halo vertex that is not trimmed (global degrees) stays,
    // even without local edges -- its edges may live on other ranks (halo.cuh)
    if (g.hpos && !alive && r.live && g.hpos[i] >= 0 && !(TRIM && trimmed(kio, (int)i))) alive = 1;
    kept = r.valid ? kio[i].y : 0;                      // kept (pre-trim) out-degree, chunks included
    const int sa = warp_sum(alive), so = warp_sum(nout), si = warp_sum(nin), sk = warp_sum(kept);
    if (lane == 0) wsum[i >> 5] = make_int4(sa, so, si, sk);
}

// k_compact_count for the keep-word layout (no FOUR): a warp counts 64 consecutive vertices,
// lane l taking l and l + 32, with the loads of both vertices -- keep word, row offsets,
// signatures, then the far ends of their kept entries, then the far ends' keep words -- issued
// together (the one-vertex form stalls on those dependent gathers, ncu: 35% of DRAM peak).  Up
// to CNT2_E kept entries per vertex go through the overlapped path (a tet mesh has at most 4
// in + out), the rest through trim_mask.  Same outputs as k_compact_count<FIRST, TRIM, false,
// true>: the trimmed survivor masks in the keep word, per-32-vertex totals (rows < nw).
constexpr int CNT2 = 2, CNT2_E = 4;
template <bool FIRST, bool TRIM>
static __global__ void __launch_bounds__(TPB_COMPACT, 6) k_compact_count2(WGraph g, const int32_t* __restrict__ cin,
                                                                         const int32_t* __restrict__ cout,
                                                                         uint32_t* __restrict__ kw, int4* __restrict__ wsum,
                                                                         int64_t nw) {
    const int lane = threadIdx.x & 31;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t wb = (t - lane) * CNT2;             // the warp's first vertex
    if ((wb >> 5) >= nw) return;                       // (warp-uniform)
    const int na = g.na;
    uint32_t w[CNT2];
    int ob[CNT2], ib[CNT2];
    bool live[CNT2];
#pragma unroll
    for (int k = 0; k < CNT2; k++) {
        const int64_t i = wb + 32 * k + lane;
        const bool ok = i < na;
        w[k] = ok ? kw[i] : 0u;
        ob[k] = ok ? __ldg(g.optr + i) : 0;
        ib[k] = ok ? __ldg(g.iptr + i) : 0;
        live[k] = ok && (FIRST || __ldcg(cin + i) != __ldcg(cout + i));
    }
    unsigned so[CNT2], si[CNT2];
#pragma unroll
    for (int k = 0; k < CNT2; k++) {
        so[k] = (w[k] >> 16) & 0xFFu;
        si[k] = w[k] >> 24;
        if (!live[k]) so[k] = si[k] = 0;
    }
    if (TRIM) {
        // far ends of the first CNT2_E kept entries of each vertex (out-row bits first)
        int x[CNT2][CNT2_E];
        unsigned rest[CNT2];
#pragma unroll
        for (int k = 0; k < CNT2; k++) {
            const bool go = live[k] && (w[k] & 0xFFu) && (w[k] & 0xFF00u);
            unsigned m = go ? (so[k] | si[k] << 8) : 0u;
#pragma unroll
            for (int q = 0; q < CNT2_E; q++) {
                x[k][q] = -1;
                if (m) {
                    const int b = __ffs(m) - 1;
                    m &= m - 1;
                    x[k][q] = b < 8 ? __ldg(g.oadj + ob[k] + b) : __ldg(g.iadj + ib[k] + (b - 8));
                }
            }
            rest[k] = m;
            if (!go) so[k] = si[k] = 0;
        }
        uint32_t y[CNT2][CNT2_E];
#pragma unroll
        for (int k = 0; k < CNT2; k++)
#pragma unroll
            for (int q = 0; q < CNT2_E; q++) y[k][q] = x[k][q] >= 0 ? __ldg(kw + x[k][q]) : 0x0101u;
#pragma unroll
        for (int k = 0; k < CNT2; k++) {
            // the entries behind x[k][q], in the same order: clear the trimmed ones
            unsigned m = so[k] | si[k] << 8, keep = m;
#pragma unroll
            for (int q = 0; q < CNT2_E; q++) {
                if (!m) break;
                const int b = __ffs(m) - 1;
                m &= m - 1;
                if (((y[k][q] & 0xFFu) == 0) | ((y[k][q] & 0xFF00u) == 0)) keep &= ~(1u << b);
            }
            if (rest[k]) {                                // more kept entries than CNT2_E
                const unsigned ro = rest[k] & 0xFFu, ri = rest[k] >> 8;
                const unsigned to = trim_mask<true>(g.oadj, ob[k], ro, 0, nullptr, kw);
                const unsigned ti = trim_mask<true>(g.iadj, ib[k], ri, 0, nullptr, kw);
                keep = (keep & ~rest[k]) | to | ti << 8;
            }
            so[k] = keep & 0xFFu;
            si[k] = keep >> 8;
            const int64_t i = wb + 32 * k + lane;
            if (i < na) kw[i] = (w[k] & 0xFFFFu) | so[k] << 16 | si[k] << 24;
        }
    }
#pragma unroll
    for (int k = 0; k < CNT2; k++) {
        const int nout = __popc(so[k]), nin = __popc(si[k]);
        const int alive = (nout + nin) > 0, kept = (int)((w[k] >> 8) & 0xFFu);
        const int sa = warp_sum(alive), so_ = warp_sum(nout), si_ = warp_sum(nin), sk = warp_sum(kept);
        const int64_t r = (wb + 32 * k) >> 5;
        if (lane == 0 && r < nw) wsum[r] = make_int4(sa, so_, si_, sk);
    }
}

// Trim-2 (McLendon; reading 17), one round on the kept graph together with
// Trim-1: an unfinished vertex i whose only kept in-edge entry comes from w, while w's only
// kept in-edge entry comes from i (i -> w kept, kin(w) == 1) -- or the same with out-edges --
// forms the SCC {i, w}.  Light rows read the kept entries from the Phase-3 bit masks; long
// rows are walked with the keep predicate (a row with exactly one kept entry).  t2[i] = w
// or -1.  k_trim2_apply then zeroes the pair's kept in-degree, so the Trim-1 test of the
// compaction removes both and their edges (the kept out-degree, which the kept-edge count
// of the trace sums, is untouched).
template <bool FIRST, typename P>
__device__ __forceinline__ int kept_single(const int32_t* __restrict__ adj, int rb, int re, unsigned m, P pred) {
    if (re - rb <= HEAVY) return m ? __ldg(adj + rb + __ffs(m) - 1) : -1;
    for (int e = rb; e < re; e++) {
        const int x = __ldg(adj + e);
        if (pred(x)) return x;
    }
    return -1;
}
template <bool FIRST, typename P>
__device__ __forceinline__ bool kept_has(const int32_t* __restrict__ adj, int rb, int re, unsigned m, P pred, int w) {
    if (re - rb <= HEAVY) {
        for (; m; m &= m - 1)
            if (__ldg(adj + rb + __ffs(m) - 1) == w) return true;
        return false;
    }
    for (int e = rb; e < re; e++)
        if (__ldg(adj + e) == w && pred(w)) return true;
    return false;
}
template <bool FIRST, bool FOUR>
static __global__ void k_trim2_find(WGraph g, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                    const int2* __restrict__ kio, const uint2* __restrict__ emask, int32_t* __restrict__ t2) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= g.na) return;
    const RowCtx r = load_row<FIRST, FOUR>(g, i, cin, cout);
    int w = -1;
    if (r.live) {
        KeepPred<FIRST, FOUR> pred{(int)i, r.a, r.b, cin, cout, g.sig2, r.c, r.d, g.min_in, g.min_out};
        const int2 k = kio[i];
        const uint2 m = emask[i];
        if (k.x == 1) {                                  // in-pattern
            const int u = kept_single<FIRST>(g.iadj, r.ib, r.ie, m.y, pred);
            if (u >= 0 && __ldg(&kio[u].x) == 1 && kept_has<FIRST>(g.oadj, r.ob, r.oe, m.x, pred, u)) w = u;
        }
        if (w < 0 && k.y == 1) {                         // out-pattern
            const int u = kept_single<FIRST>(g.oadj, r.ob, r.oe, m.x, pred);
            if (u >= 0 && __ldg(&kio[u].y) == 1 && kept_has<FIRST>(g.iadj, r.ib, r.ie, m.y, pred, u)) w = u;
        }
    }
    t2[i] = w;
}
static __global__ void k_trim2_apply(int32_t na, const int32_t* __restrict__ t2, int2* __restrict__ kio) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < na && t2[i] >= 0) kio[i].x = 0;
}

// the optional outputs of k_compact_map
struct MapExtra {
    int32_t *min_in2, *min_out2;     // 4-signature variant: the minimum pair of the next graph
    const int32_t* t2;               // Trim-2 partners (labels of the pairs)
    const int2* kio;                 // kept degrees (partitioned mode: trimmed halo vertices)
    int trim;
    int32_t* hpos2;                  // partitioned mode: halo positions of the next graph
    int32_t lab_lo, lab_hi;          // labels written only for IDs in [lab_lo, lab_hi)
    int32_t* slot;                   // priority -> local index of the next graph, or nullptr
};

// New numbering, Phase 1 reset of the survivors (rule R2), final labels of
// the vertices that leave, new offsets, heavy-row chunk list.
// Survivors restart from their priority pi(v) (reading 16).  A finished vertex leaves
// with its signature s = max priority of its SCC; with raw IDs that is the label itself,
// otherwise it is stored as -(s+1) and k_relabel_* turn it into the SCC's max vertex ID.
template <bool FIRST, bool KW = false>
static __global__ void __launch_bounds__(TPB_COMPACT, 8) k_compact_map(WGraph g, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                              const int2* __restrict__ cnt, const int4* __restrict__ wscan,
                              const int4* __restrict__ totals, int32_t* __restrict__ newidx,
                              int32_t* __restrict__ act2, int32_t* __restrict__ cin2, int32_t* __restrict__ cout2,
                              int32_t* __restrict__ optr2, int32_t* __restrict__ iptr2, int32_t* __restrict__ labels,
                              Chunk* __restrict__ chunks, int* __restrict__ nchunks, int chunk_cap, Prio P,
                              const int32_t* __restrict__ orig, PackOut pk, MapExtra X) {
    int32_t* __restrict__ min_in2 = X.min_in2;
    int32_t* __restrict__ min_out2 = X.min_out2;
    const int32_t* __restrict__ t2 = X.t2;
    const int2* __restrict__ kio = X.kio;
    const int trim = X.trim;
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i == 0) {
        const int4 t = *totals;
        optr2[t.x] = t.y;
        iptr2[t.x] = t.z;
    }
    if (pk.pnin) {                         // pack: empty slot words past the last vertex of the last tile
        const int na2 = totals->x;
        const int pad_end = (na2 + TILE - 1) & ~(TILE - 1);
        for (int64_t k = na2 + i; k < pad_end; k += (int64_t)gridDim.x * blockDim.x) {
            pk.pnin[k] = PK_EMPTY;
            pk.pnout[k] = PK_EMPTY;
        }
    }
    const bool valid = i < g.na;
    int2 c = make_int2(0, 0);
    if (valid && KW) {                                 // the survivor masks of the keep word
        const uint32_t w = ((const uint32_t*)cnt)[i];
        c = make_int2(__popc((w >> 16) & 0xFFu), __popc(w >> 24));
    } else if (valid) {
        c = cnt[i];
    }
    int alive = (c.x + c.y) > 0;
    if (g.hpos && valid && !alive && g.hpos[i] >= 0 && (FIRST || cin[i] != cout[i]) && !(trim && trimmed(kio, (int)i)))
        alive = 1;                                     // (the same rule as k_compact_count)
    const int4 base = wscan[i >> 5];
    int j, po, pi;
    if (KW) {      // degrees <= KW_DEG: the three warp prefixes packed into one scan (6 + 10 + 10 bits)
        const int pk = alive | c.x << 6 | c.y << 16;
        const int ex = warp_incl_scan(pk, lane) - pk;
        j = (ex & 63) + base.x;
        po = ((ex >> 6) & 1023) + base.y;
        pi = ((ex >> 16) & 1023) + base.z;
    } else {
        j = warp_incl_scan(alive, lane) - alive + base.x;
        po = warp_incl_scan(c.x, lane) - c.x + base.y;
        pi = warp_incl_scan(c.y, lane) - c.y + base.z;
    }
    if (!valid) return;
    const int v = g.act ? g.act[i] : (int)i;          // storage ID
    const int ov = orig ? orig[v] : v;                 // caller's ID (reorder.cuh)
    if (alive) {
        newidx[i] = j;
        act2[j] = v;
        if (pk.pnin && (j & (TILE - 1)) == 0) pk.ext_cnt[j / TILE] = 0;   // the tile's cut-edge count
        const int pv = (int)prio_of(P, (uint32_t)ov);
        cin2[j] = pv;       // Phase 1: v_in <- v_id, v_out <- v_id for the unfinished
        cout2[j] = pv;
        if (X.hpos2) X.hpos2[j] = g.hpos[i];
        if (X.slot) X.slot[pv] = j;  // priority -> local index (ECL_SCC_COMPRESS / ECL_SCC_RAISE)
        if (min_in2) {      // the minimum pair restarts from the vertex too
            min_in2[j] = mirror_prio(pv);
            min_out2[j] = mirror_prio(pv);
        }
        optr2[j] = po;
        iptr2[j] = pi;
        for (int dir = 0; dir < 2; dir++) {
            const int deg = dir ? c.y : c.x, beg = dir ? pi : po;
            if (deg > HEAVY_T) {
                const int nc = (deg + CHUNK - 1) / CHUNK;
                const int at = atomicAdd(nchunks, nc);
                for (int k = 0; k < nc && at + k < chunk_cap; k++)
                    chunks[at + k] = Chunk{j, dir, beg + k * CHUNK, min(beg + (k + 1) * CHUNK, beg + deg), at};
            }
        }
    } else {
        newidx[i] = -1;
        int lab = ov;   // unfinished (or trimmed) and edgeless: a singleton SCC
        if (!FIRST) {
            const int a = cin[i], b = cout[i];
            if (a == b) lab = P.ids ? a : -(a + 1);
        }
        if (t2 && t2[i] >= 0) {      // Trim-2 pair {v, w}: named by its larger member
            const int w = t2[i];
            const int vw = g.act ? g.act[w] : w;
            const int ow = orig ? orig[vw] : vw;
            lab = P.ids ? max(ov, ow) : -((int)max(prio_of(P, (uint32_t)ov), prio_of(P, (uint32_t)ow)) + 1);
        }
        if (ov >= X.lab_lo && ov < X.lab_hi) labels[ov] = lab;    // partitioned: the owner writes
    }
}

// k_compact_map for the keep-word layout (rows <= KW_DEG, no FOUR / TRIM2): a warp maps 128
// consecutive vertices, lane l taking l, l + 32, l + 64, l + 96, so each thread has four
// independent coalesced loads of keep words (and IDs, and signatures) in flight instead of one
// -- the one-vertex form stalls on those streaming loads (ncu: 35% of DRAM peak, most stall
// samples at the keep-word and ID loads) -- while every store stays a coalesced warp row.
// Same outputs as k_compact_map<FIRST, true>.  The warp's 128 vertices are 4 scan warps of
// k_compact_count: row k's base is wscan of its first vertex.
constexpr int MAP4 = 4;
template <bool FIRST>
static __global__ void __launch_bounds__(TPB_COMPACT, 6) k_compact_map4(WGraph g, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                              const uint32_t* __restrict__ kw, const int4* __restrict__ wscan,
                              const int4* __restrict__ totals, int32_t* __restrict__ newidx,
                              int32_t* __restrict__ act2, int32_t* __restrict__ cin2, int32_t* __restrict__ cout2,
                              int32_t* __restrict__ optr2, int32_t* __restrict__ iptr2, int32_t* __restrict__ labels,
                              Prio P, const int32_t* __restrict__ orig, PackOut pk, MapExtra X) {
    const int lane = threadIdx.x & 31;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t wb = (t - lane) * MAP4;              // the warp's first vertex
    if (t == 0) {
        const int4 tt = *totals;
        optr2[tt.x] = tt.y;
        iptr2[tt.x] = tt.z;
    }
    if (pk.pnin) {                         // pack: empty slot words past the last vertex of the last tile
        const int na2 = totals->x;
        const int pad_end = (na2 + TILE - 1) & ~(TILE - 1);
        for (int64_t k = na2 + t; k < pad_end; k += (int64_t)gridDim.x * blockDim.x) {
            pk.pnin[k] = PK_EMPTY;
            pk.pnout[k] = PK_EMPTY;
        }
    }
    const int na = g.na;
    if (wb >= na) return;                              // (warp-uniform)
    uint32_t w[MAP4];
    int sa[MAP4], sb[MAP4], av[MAP4];
#pragma unroll
    for (int k = 0; k < MAP4; k++) {
        const int64_t i = wb + 32 * k + lane;
        const bool ok = i < na;
        w[k] = ok ? __ldg(kw + i) : 0u;
        av[k] = g.act ? (ok ? __ldg(g.act + i) : 0) : (int)i;
        if (!FIRST) { sa[k] = ok ? __ldcg(cin + i) : 0; sb[k] = ok ? __ldcg(cout + i) : 0; }
    }
#pragma unroll
    for (int k = 0; k < MAP4; k++) {
        const int64_t i = wb + 32 * k + lane;
        if (wb + 32 * k >= na) break;                  // (warp-uniform)
        const bool ok = i < na;
        const int co = __popc((w[k] >> 16) & 0xFFu), ci = __popc(w[k] >> 24);
        int al = (co + ci) > 0;
        if (g.hpos && ok && !al && g.hpos[i] >= 0 && (FIRST || sa[k] != sb[k]) && !(X.trim && trimmed(X.kio, (int)i)))
            al = 1;
        const int4 base = wscan[(wb + 32 * k) >> 5];
        const int pk_ = al | co << 8 | ci << 19;       // per scan warp: alive <= 32, degrees <= 256
        const int ex = warp_incl_scan(pk_, lane) - pk_;
        if (!ok) continue;
        const int j = (ex & 0xFF) + base.x, po = ((ex >> 8) & 0x7FF) + base.y, pi = ((ex >> 19) & 0x7FF) + base.z;
        const int v = av[k];
        const int ov = orig ? orig[v] : v;
        if (al) {
            newidx[i] = j;
            act2[j] = v;
            if (pk.pnin && (j & (TILE - 1)) == 0) pk.ext_cnt[j / TILE] = 0;
            const int pv = (int)prio_of(P, (uint32_t)ov);
            cin2[j] = pv;       // Phase 1: v_in <- v_id, v_out <- v_id for the unfinished
            cout2[j] = pv;
            if (X.hpos2) X.hpos2[j] = g.hpos[i];
            if (X.slot) X.slot[pv] = j;
            optr2[j] = po;
            iptr2[j] = pi;
        } else {
            newidx[i] = -1;
            int lab = ov;      // unfinished (or trimmed) and edgeless: a singleton SCC
            if (!FIRST && sa[k] == sb[k]) lab = P.ids ? sa[k] : -(sa[k] + 1);
            if (ov >= X.lab_lo && ov < X.lab_hi) labels[ov] = lab;
        }
    }
}

// Final labels under priorities: an SCC is named by s = max priority; its label is the
// largest vertex ID with signature s: the slots (cleared to -1) take the max ID of every
// signature (fold: lanes with the same slot grouped first, so a giant SCC costs one atomic
// per warp), then every finished vertex reads its slot (apply).
static __global__ void k_relabel_fold(int32_t n, const int32_t* __restrict__ labels, int32_t* __restrict__ slot) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t start = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t v0 = start - (threadIdx.x & 31); v0 < n; v0 += stride) {
        const int64_t v = v0 + (threadIdx.x & 31);
        int key = -1;
        if (v < n) {
            const int l = labels[v];
            if (l < 0) key = -l - 1;
        }
        if (!__any_sync(FULL, key >= 0)) continue;
        const unsigned grp = __match_any_sync(FULL, key);
        // lanes hold increasing v: the group's last lane has its largest ID
        if (key >= 0 && (threadIdx.x & 31) == 31 - __clz(grp)) atomicMax(slot + key, (int)v);
    }
}
static __global__ void k_relabel_apply(int32_t n, int32_t* __restrict__ labels, const int32_t* __restrict__ slot) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int l = labels[v];
        if (l < 0) labels[v] = slot[-l - 1];
    }
}
// debug snapshot of the vertices that already left: their (in, out) in priority space
static __global__ void k_snapshot_left(int32_t n, const int32_t* __restrict__ labels, int32_t* __restrict__ din,
                                int32_t* __restrict__ dout, Prio P) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int l = labels[v];
        const int s = l < 0 ? -l - 1 : (int)prio_of(P, (uint32_t)l);
        din[v] = s;
        dout[v] = s;
    }
}

// write one row's survivors (as new local indices) starting at dst[pos]
template <typename P>
__device__ __forceinline__ void emit_row(const int32_t* __restrict__ adj, int rb, int re, bool go, int pos,
                                         const int32_t* __restrict__ newidx, int32_t* __restrict__ dst, int lane,
                                         P pred, bool chunked = false, bool light = true) {
    if (chunked && re - rb > HEAVY_T) go = false;      // long row: k_scatter_chunks writes it
    if (light && go && re - rb <= HEAVY) {
        for (int e = rb; e < re; e++) {
            const int x = __ldg(adj + e);
            if (pred(x)) dst[pos++] = __ldg(newidx + x);
        }
    }
    unsigned hm = __ballot_sync(FULL, go && re - rb > HEAVY);
    while (hm) {
        const int src = __ffs(hm) - 1;
        hm &= hm - 1;
        const int sb = __shfl_sync(FULL, rb, src), se = __shfl_sync(FULL, re, src);
        int spos = __shfl_sync(FULL, pos, src);
        const P bp = pred.bcast(src);
        for (int base = sb; base < se; base += WARP) {
            const int e = base + lane;
            int x = 0;
            if (e < se) x = __ldg(adj + e);
            const bool k = (e < se) && bp(x);
            const unsigned bm = __ballot_sync(FULL, k);
            if (k) dst[spos + __popc(bm & ((1u << lane) - 1))] = __ldg(newidx + x);
            spos += __popc(bm);
        }
    }
}

template <bool FIRST, bool TRIM, bool FOUR, bool KW = false>
static __global__ void k_compact_scatter(WGraph g, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                  const int2* __restrict__ kio, const int32_t* __restrict__ newidx, const int32_t* __restrict__ optr2,
                                  const int32_t* __restrict__ iptr2, int32_t* __restrict__ oadj2,
                                  int32_t* __restrict__ iadj2, int chunked, const uint2* __restrict__ emask,
                                  PackOut pk) {
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const RowCtx r = load_row<FIRST, FOUR>(g, i, cin, cout);
    const int j = r.valid ? newidx[i] : -1;
    const bool go = j >= 0;
    int po = 0, pi = 0, ncut = 0;
    uint2 sm = make_uint2(0, 0);
    bool lo = false, li = false;
    if (go) {
        po = optr2[j];
        pi = iptr2[j];
        if (KW) {                                      // light rows: the survivors' bits
            const uint32_t w = ((const uint32_t*)emask)[i];
            sm = make_uint2((w >> 16) & 0xFFu, w >> 24);
        } else {
            sm = emask[i];
        }
        lo = r.oe - r.ob <= HEAVY;
        li = r.ie - r.ib <= HEAVY;
        if (pk.pnin) {
            if (!(lo && li)) *pk.bad = 1;              // a warp-path row: k_tile_pack rebuilds the pack
            const int tb = j & ~(TILE - 1);
            if (lo) pk.pnout[j] = emit_mask_pack(g.oadj, r.ob, sm.x, (int)i, newidx, oadj2, po, tb, ncut);
            if (li) pk.pnin[j] = emit_mask_pack(g.iadj, r.ib, sm.y, (int)i, newidx, iadj2, pi, tb, ncut);
        } else {
            if (lo) emit_mask(g.oadj, r.ob, sm.x, (int)i, newidx, oadj2, po);
            if (li) emit_mask(g.iadj, r.ib, sm.y, (int)i, newidx, iadj2, pi);
        }
    }
    if (pk.pnin) {
        // cut edges: lanes of one tile reserve their slots with one atomic per warp and tile
        const int tile = go ? j / TILE : -1;
        const unsigned grp = __match_any_sync(FULL, tile);
        const int leader = __ffs(grp) - 1;
        // alive lanes hold increasing j, so between two lanes of one tile there are only lanes
        // of that tile or dead ones (ncut 0): the offset is an exclusive warp scan relative to
        // the group's leader
        const int excl = warp_incl_scan(ncut, lane) - ncut;
        const int pre = excl - __shfl_sync(FULL, excl, leader);
        const int tot = __reduce_add_sync(grp, ncut);
        int base = 0;
        if (go && lane == leader && tot) base = atomicAdd(pk.ext_cnt + tile, tot);
        base = __shfl_sync(FULL, base, leader);
        if (go && ncut) {
            const int tb = j & ~(TILE - 1);
            int2* E = pk.ext + (int64_t)__ldg(optr2 + tb) + __ldg(iptr2 + tb);
            int at = base + pre;
            if (lo) emit_cut(g.oadj, r.ob, sm.x, newidx, j, tb, PK_DIR, E, at);
            if (li) emit_cut(g.iadj, r.ib, sm.y, newidx, j, tb, 0, E, at);
        }
    }
    if (KW) return;                                    // (no row longer than HEAVY)
    SurvivePred<FIRST, TRIM, FOUR> pred{(int)i, r.a, r.b, cin, cout, kio, g.sig2, r.c, r.d, g.min_in, g.min_out};
    emit_row(g.oadj, r.ob, r.oe, go, po, newidx, oadj2, lane, pred, chunked, false);
    emit_row(g.iadj, r.ib, r.ie, go, pi, newidx, iadj2, lane, pred, chunked, false);
}

// ------------------------------------------------------------------ long rows in chunks
// Rows longer than HEAVY_T are split into CHUNK-edge pieces (one warp each) in every
// compaction kernel, so a 100k-edge hub costs 200 warps, not one.  Counts are folded in
// with atomics; the scatter places a chunk after the survivors of the earlier chunks of
// its row (chunk_cnt prefix), so rows stay stable.
template <bool FIRST, bool FOUR>
static __global__ void __launch_bounds__(256) k_keep_chunks(WGraph g, const Chunk* __restrict__ chunks, int nchunks,
                                                            const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                                            int2* __restrict__ kio) {
    const int lane = threadIdx.x & 31;
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const Chunk k = chunks[c];
    const int a = FIRST ? 0 : cin[k.i], b = FIRST ? 0 : cout[k.i];
    if (!FIRST && a == b) return;                        // finished owner keeps nothing
    const int mc = !FIRST && FOUR ? g.min_in[k.i] : 0, md = !FIRST && FOUR ? g.min_out[k.i] : 0;
    const int32_t* adj = k.dir ? g.iadj : g.oadj;
    int cc = 0;
    for (int e = k.beg + lane; e < k.end; e += WARP)
        cc += keep_edge<FIRST, FOUR>(k.i, a, b, __ldg(adj + e), cin, cout, g.sig2, mc, md, g.min_in, g.min_out);
    cc = warp_sum(cc);
    if (lane == 0 && cc) {
        atomicAdd(k.dir ? &kio[k.i].x : &kio[k.i].y, cc);
    }
}
template <bool FIRST, bool TRIM, bool FOUR>
static __global__ void __launch_bounds__(256) k_count_chunks(WGraph g, const Chunk* __restrict__ chunks, int nchunks,
                                                             const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                                             const int2* __restrict__ kio,
                                                             int* __restrict__ chunk_cnt, int2* __restrict__ hcnt) {
    const int lane = threadIdx.x & 31;
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const Chunk k = chunks[c];
    const int a = FIRST ? 0 : cin[k.i], b = FIRST ? 0 : cout[k.i];
    int cc = 0;
    if ((FIRST || a != b) && !(TRIM && trimmed(kio, k.i))) {
        const int32_t* adj = k.dir ? g.iadj : g.oadj;
        const int mc = !FIRST && FOUR ? g.min_in[k.i] : 0, md = !FIRST && FOUR ? g.min_out[k.i] : 0;
        SurvivePred<FIRST, TRIM, FOUR> pred{k.i, a, b, cin, cout, kio, g.sig2, mc, md, g.min_in, g.min_out};
        for (int e = k.beg + lane; e < k.end; e += WARP) cc += pred(__ldg(adj + e));
        cc = warp_sum(cc);
    }
    if (lane == 0) {
        chunk_cnt[c] = cc;
        if (cc) atomicAdd(k.dir ? &hcnt[k.i].y : &hcnt[k.i].x, cc);
    }
}
template <bool FIRST, bool TRIM, bool FOUR>
static __global__ void __launch_bounds__(256) k_scatter_chunks(WGraph g, const Chunk* __restrict__ chunks, int nchunks,
                                                               const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                                               const int2* __restrict__ kio,
                                                               const int* __restrict__ chunk_cnt,
                                                               const int32_t* __restrict__ newidx,
                                                               const int32_t* __restrict__ optr2, const int32_t* __restrict__ iptr2,
                                                               int32_t* __restrict__ oadj2, int32_t* __restrict__ iadj2) {
    const int lane = threadIdx.x & 31;
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const Chunk k = chunks[c];
    if (chunk_cnt[c] == 0) return;
    const int j = newidx[k.i];
    // survivors of the earlier chunks of this row
    int before = 0;
    for (int q = k.first + lane; q < (int)c; q += WARP) before += chunk_cnt[q];
    before = warp_sum(before);
    int pos = (k.dir ? iptr2[j] : optr2[j]) + before;
    const int a = FIRST ? 0 : cin[k.i], b = FIRST ? 0 : cout[k.i];
    const int32_t* adj = k.dir ? g.iadj : g.oadj;
    int32_t* dst = k.dir ? iadj2 : oadj2;
    const int mc = !FIRST && FOUR ? g.min_in[k.i] : 0, md = !FIRST && FOUR ? g.min_out[k.i] : 0;
    SurvivePred<FIRST, TRIM, FOUR> pred{k.i, a, b, cin, cout, kio, g.sig2, mc, md, g.min_in, g.min_out};
    for (int base = k.beg; base < k.end; base += WARP) {
        const int e = base + lane;
        int x = 0;
        if (e < k.end) x = __ldg(adj + e);
        const bool keep = (e < k.end) && pred(x);
        const unsigned bm = __ballot_sync(FULL, keep);
        if (keep) dst[pos + __popc(bm & ((1u << lane) - 1))] = __ldg(newidx + x);
        pos += __popc(bm);
    }
}
// chunk list of the input graph (CSR rows from row_ptr, CSC rows from iptr)
// (and the largest row of either direction, for the small-degree compaction)
static __global__ void k_ingest_chunks(int32_t n, const int32_t* __restrict__ ptr, int dir, Chunk* __restrict__ chunks,
                                       int* __restrict__ nchunks, int chunk_cap, int* __restrict__ maxdeg) {
    __shared__ int s_md;
    const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int beg = v < n ? ptr[v] : 0, deg = v < n ? ptr[v + 1] - beg : 0;
    if (threadIdx.x == 0) s_md = 0;
    __syncthreads();
    const int md = __reduce_max_sync(FULL, deg);
    if ((threadIdx.x & 31) == 0 && md) atomicMax(&s_md, md);
    __syncthreads();
    // one global atomic per block, and only while it raises the maximum (the blocks of a
    // launch all target one address)
    if (threadIdx.x == 0 && s_md > *(volatile int*)maxdeg) atomicMax(maxdeg, s_md);
    if (v >= n || deg <= HEAVY_T) return;
    const int nc = (deg + CHUNK - 1) / CHUNK;
    const int at = atomicAdd(nchunks, nc);
    for (int k = 0; k < nc && at + k < chunk_cap; k++)
        chunks[at + k] = Chunk{(int32_t)v, dir, beg + k * CHUNK, min(beg + (k + 1) * CHUNK, beg + deg), at};
}
// CSC scatter of long CSR rows (input graph)
template <bool RANK>
static __global__ void __launch_bounds__(256) k_csc_scatter_chunks(const Chunk* __restrict__ chunks, int nchunks,
                                                                   const int32_t* __restrict__ ci, const int32_t* __restrict__ iptr,
                                                                   const int32_t* __restrict__ rank, int32_t* cursor,
                                                                   int32_t* __restrict__ iadj) {
    const int lane = threadIdx.x & 31;
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const Chunk k = chunks[c];
    if (k.dir) return;
    for (int e = k.beg + lane; e < k.end; e += WARP) {
        const int w = __ldg(ci + e);
        iadj[__ldg(iptr + w) + csc_slot<RANK>(rank, cursor, e, w)] = k.i;
    }
}

// ------------------------------------------------------------------ Phase 2
// Pass protocol (shared by the kernels of one pass; `first` marks the first kernel of
// the pass): pass p clears changed[p+1]; all kernels of pass p return at once if pass
// p-1 changed nothing; a kernel sets changed[p] if it raised any signature.  A pass that
// changes nothing observed a consistent snapshot and so certifies the fixed point.
__device__ __forceinline__ bool pass_begin(DevCounters* dc, int pass, bool first) {
    if (first && blockIdx.x == 0 && threadIdx.x == 0) dc->changed[(pass + 1) & (RING - 1)] = 0;
    if (pass > 0 && ld_vol(&dc->changed[(pass - 1) & (RING - 1)]) == 0) return false;
    if (first && blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(&dc->passes, 1ull);
    return true;
}

// Heavy rows: one warp per chunk of a long row; the chunk max is folded in with
// atomicMax (monotone, so concurrent chunks of one row commute).
static __global__ void __launch_bounds__(256) k_prop_heavy(const Chunk* __restrict__ chunks, int nchunks, WGraph g,
                                                    int32_t* __restrict__ cin, int32_t* __restrict__ cout,
                                                    DevCounters* __restrict__ dc, int pass) {
    if (!pass_begin(dc, pass, true)) return;
    const int lane = threadIdx.x & 31;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    bool ch = false;
    long long ne = 0;                              // edges reduced by this warp (accounting)
    for (int64_t c = wid; c < nchunks; c += nw) {
        const Chunk k = chunks[c];
        const int32_t* adj = k.dir ? g.iadj : g.oadj;
        int32_t* sig = k.dir ? cin : cout;
        int acc = 0;
        for (int e = k.beg + lane; e < k.end; e += WARP) acc = max(acc, ld_cg(sig + __ldg(adj + e)));
        acc = warp_max(acc);
        ne += k.end - k.beg;
        if (lane == 0 && acc > ld_cg(sig + k.i)) {
            if (atomicMax(sig + k.i, acc) < acc) ch = true;
        }
    }
    if (lane == 0 && ne) atomicAdd(&dc->heavy_e, (unsigned long long)ne);
    if (__any_sync(FULL, ch) && lane == 0) dc->changed[pass & (RING - 1)] = 1;
}

// Block-local fixed point ("every thread block internally iterates until none of
// the edges assigned to it propagate any more values").  CTA = tile of TILE consecutive
// local vertices; thread t owns vertices 4t..4t+3 of the tile.  Each visit:
//   1. gather the out-of-tile neighbours from global memory (Alg. 1 l.10-11, pull:
//      in[v] <- max in[u] over in-edges, out[v] <- max out[w] over out-edges) and cache
//      the intra-tile neighbours as 16-bit slots in shared memory;
//   2. frontier propagation in shared memory: a vertex whose value rose pushes it to its
//      intra-tile dependents (in along out-edges, out along in-edges) with shared-memory
//      atomicMax, and a dependent that rose is flagged.  Each warp keeps draining the
//      flags of its own 128 vertices (atomic fetch-and-clear) so chains inside a warp's
//      region need no block barrier; block rounds repeat until a round does no work.
//      Work is proportional to the number of raises, not to rounds x tile size;
//   3. write raised signatures back and flag the out-of-tile dependents' tiles dirty.
// Rows longer than HEAVY_T are skipped here (k_prop_heavy folds them in).  Tile order
// alternates with the pass parity so values can ride the block schedule both ways.
// full: every vertex starts flagged and step 1 also pulls the intra-tile neighbours'
// values (first visit of a phase, and every visit when heavy rows exist: an intra-tile
// edge whose source row is heavy is not in any push list, so it is covered by the pull).
// SYNC = ablation: no step 2 (one relaxation per pass, "separate kernels").
#ifdef ECL_PROF
#define PROF_ADD(dc, k, v) atomicAdd(&(dc)->prof[k], (unsigned long long)(v))
#else
#define PROF_ADD(dc, k, v) ((void)0)
#endif
constexpr int SLOTS = 4;                 // cached intra-tile neighbours per vertex and direction
constexpr uint16_t NOSLOT = 0xFFFF;
template <int TT>
constexpr size_t tile_dyn_smem() { return (size_t)TT * (4 + 4 + 8 + 8); }   // values + slots

// slots are packed 4 x 16 bit in a 64-bit word (NOSLOT = empty).  A raised target w is
// flagged in its owner's flag word (thread w/4 owns byte w%4).
__device__ __forceinline__ void flag_set(unsigned* __restrict__ fw, unsigned w) {
    atomicOr(fw + (w >> 2), 1u << (8 * (w & 3)));
}
__device__ __forceinline__ void push_slots(unsigned long long nb, int val, int* __restrict__ sig,
                                           unsigned* __restrict__ fw, int& any) {
#pragma unroll
    for (int q = 0; q < SLOTS; q++) {
        unsigned w = (unsigned)(nb >> (16 * q)) & 0xFFFFu;
        if (w == NOSLOT) break;
        w &= 0x7FFFu;                                  // slot 3 may carry the SLOW mark
        if (sig[w] < val && atomicMax(sig + w, val) < val) { flag_set(fw, w); any = 1; }
    }
}
__device__ __forceinline__ void add_slot(unsigned long long& pk, int& ns, unsigned idx) {
    pk &= ~(0xFFFFull << (16 * ns));
    pk |= (unsigned long long)idx << (16 * ns);
    ns++;
}

// slots: SLOWBIT on slot 3 marks a vertex with more than SLOTS intra-tile neighbours in
// that direction (it walks its global row for the rest)
constexpr unsigned long long SLOW_MARK = 0x8000ull << 48;

// Shared-memory working set of one tile visit (dynamic shared memory + static arrays).
template <int TT>
struct TileSmem {
    int* s_in;
    int* s_out;
    unsigned long long* s_nin;
    unsigned long long* s_nout;
    unsigned* s_fin;
    unsigned* s_fout;
    unsigned short* s_queue;      // drain item queues (k_prop_tile)
    unsigned long long* s_acc;    // pack kernels: per-CTA visited vertices / edges (thread 0), flushed once
};

// dirty marking of the tiles that depend on a raised value (pass mode: byte flags for
// the next pass)
struct MarkNext {
    uint8_t* next;
    __device__ __forceinline__ bool on() const { return next != nullptr; }
    __device__ __forceinline__ void operator()(int t) const { next[t] = 1; }
};
// flag the intra-tile vertices in slot word nb (and, for a slow row, the rest of the
// global row) for a re-pull: plain byte stores
__device__ __forceinline__ void notify(unsigned long long nb, const int32_t* __restrict__ ptr,
                                       const int32_t* __restrict__ adj, int base, int cnt, int v, uint8_t* f) {
#pragma unroll
    for (int k = 0; k < SLOTS; k++) {
        const unsigned w = (unsigned)(nb >> (16 * k)) & 0xFFFFu;
        if (w == NOSLOT) break;
        ((volatile uint8_t*)f)[w & 0x7FFFu] = 1;
    }
    if ((nb & SLOW_MARK) && (nb >> 48) != 0xFFFFull)
        for (int e = __ldg(ptr + base + v), ee = __ldg(ptr + base + v + 1); e < ee; e++) {
            const int w = __ldg(adj + e) - base;
            if ((unsigned)w < (unsigned)cnt) ((volatile uint8_t*)f)[w] = 1;
        }
}

// Step 2 drain loop (see tile_visit): owner-computes pulls over the intra-tile slots until
// no flag is left.  Shared by the tile and the tile-pack kernels.
__device__ __forceinline__ void drain_local(const WGraph& g, int* __restrict__ s_in, int* __restrict__ s_out,
                                            const unsigned long long* __restrict__ s_nin,
                                            const unsigned long long* __restrict__ s_nout,
                                            unsigned* __restrict__ s_fin, unsigned* __restrict__ s_fout,
                                            unsigned short* __restrict__ s_queue, int base, int cnt,
                                            unsigned& prof_rounds, unsigned& prof_drains, unsigned& prof_pushes) {
    const int tid = threadIdx.x;
    const int lane = tid & 31, wq0 = (tid >> 5) * (2 * 32 * VPT);
    for (;;) {
        int worked = 0;
#ifdef ECL_PROF
        if (tid == 0) prof_rounds++;
#endif
        for (;;) {                                       // drain this warp's flags
#ifdef ECL_PROF
            if (lane == 0) prof_drains++;
#endif
            unsigned wi = ((volatile unsigned*)s_fin)[tid], wo = ((volatile unsigned*)s_fout)[tid];
            if (wi) wi = atomicExch(s_fin + tid, 0u);
            if (wo) wo = atomicExch(s_fout + tid, 0u);
            const unsigned items = ((wi & 0x01u) | ((wi >> 7) & 0x02u) | ((wi >> 14) & 0x04u) | ((wi >> 21) & 0x08u)) |
                                   (((wo & 0x01u) | ((wo >> 7) & 0x02u) | ((wo >> 14) & 0x04u) | ((wo >> 21) & 0x08u)) << 4);
            const int c = __popc(items);
            const int incl = warp_incl_scan(c, lane);
            const int total = __shfl_sync(FULL, incl, 31);
            if (total == 0) break;                       // region drained
            worked = 1;
#ifdef ECL_PROF
            prof_pushes += c;
#endif
            {
                int pos = wq0 + incl - c;
                unsigned it = items;
                while (it) {
                    const int bit = __ffs(it) - 1;
                    it &= it - 1;
                    s_queue[pos++] = (unsigned short)(((tid * VPT + (bit & 3)) << 1) | (bit >> 2));
                }
            }
            __syncwarp();
            __threadfence_block();
            int any = 0;
            for (int q = lane; q < total; q += 32) {
                const unsigned item = s_queue[wq0 + q];
                const int v = (int)(item >> 1);
                const bool dir_out = item & 1u;
                int* sig = dir_out ? s_out : s_in;
                // pull: v_in from in-neighbours, v_out from out-neighbours
                const unsigned long long src = dir_out ? s_nout[v] : s_nin[v];
                const int32_t* sptr = dir_out ? g.optr : g.iptr;
                const int32_t* sadj = dir_out ? g.oadj : g.iadj;
                const int old = ((volatile int*)sig)[v];
                int val = old;
#pragma unroll
                for (int k = 0; k < SLOTS; k++) {
                    unsigned w = (unsigned)(src >> (16 * k)) & 0xFFFFu;
                    if (w == NOSLOT) break;
                    val = max(val, ((volatile int*)sig)[w & 0x7FFFu]);
                }
                if ((src & SLOW_MARK) && (src >> 48) != 0xFFFFull)
                    for (int e = __ldg(sptr + base + v), ee = __ldg(sptr + base + v + 1); e < ee; e++) {
                        const int w = __ldg(sadj + e) - base;
                        if ((unsigned)w < (unsigned)cnt) val = max(val, ((volatile int*)sig)[w]);
                    }
                if (val > old) {
                    ((volatile int*)sig)[v] = val;
                    __threadfence_block();
                    // dependents: out-neighbours re-pull v_in, in-neighbours re-pull v_out
                    if (dir_out) notify(s_nin[v], g.iptr, g.iadj, base, cnt, v, (uint8_t*)s_fout);
                    else notify(s_nout[v], g.optr, g.oadj, base, cnt, v, (uint8_t*)s_fin);
                    any = 1;
                }
            }
            __syncwarp();
            if (!__any_sync(FULL, any)) break;           // raised nothing: region drained
        }
        if (!__syncthreads_or(worked)) break;            // a round with no work: done
    }
}

// One block-local fixed point of tile `tile` (steps 1-3 above).  Returns non-zero in
// every thread if a signature was raised.
template <bool SYNC, int TT, typename Mark>
__device__ __forceinline__ int tile_visit(const WGraph& g, int32_t* __restrict__ cin, int32_t* __restrict__ cout,
                                          DevCounters* __restrict__ dc, int tile, int full, Mark mark,
                                          const TileSmem<TT>& S) {
    int* s_in = S.s_in;
    int* s_out = S.s_out;
    unsigned long long* s_nin = S.s_nin;
    unsigned long long* s_nout = S.s_nout;
    unsigned* s_fin = S.s_fin;
    unsigned* s_fout = S.s_fout;
    unsigned short* s_queue = S.s_queue;
    const int tid = threadIdx.x;
    const int base = tile * TT;
    const int cnt = min(TT, g.na - base);
#ifdef ECL_PROF
    const long long t_start = clock64();
#endif

    // ---- step 1: rows, out-of-tile pulls (global, L2-coherent), intra-tile slots
    unsigned fin = 0, fout = 0;
    int me = 0;                                   // out-edges of the visited rows (accounting)
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int v = tid * VPT + k;
        int x = 0, y = 0;
        unsigned long long ni = ~0ull, no = ~0ull;
        if (v < cnt) {
            const int gi = base + v;
            int ob = __ldg(g.optr + gi);
            const int oe = __ldg(g.optr + gi + 1);
            int ib = __ldg(g.iptr + gi);
            const int ie = __ldg(g.iptr + gi + 1);
            me += oe - ob;
            if (oe - ob > HEAVY_T) ob = oe;       // heavy: reduced by k_prop_heavy
            if (ie - ib > HEAVY_T) ib = ie;
            const int x0 = ld_cg(cin + gi), y0 = ld_cg(cout + gi);
            x = x0;
            y = y0;
            int ns = 0;
            for (int e = ib; e < ie; e++) {
                const int u = __ldg(g.iadj + e);
                if (SYNC || (unsigned)(u - base) >= (unsigned)cnt) { x = max(x, ld_cg(cin + u)); continue; }
                if (full) x = max(x, ld_cg(cin + u));   // see "full" above: heavy rows do not push
                if (ns < SLOTS) add_slot(ni, ns, (unsigned)(u - base));
                else ni |= SLOW_MARK;
            }
            ns = 0;
            for (int e = ob; e < oe; e++) {
                const int w = __ldg(g.oadj + e);
                if (SYNC || (unsigned)(w - base) >= (unsigned)cnt) { y = max(y, ld_cg(cout + w)); continue; }
                if (full) y = max(y, ld_cg(cout + w));
                if (ns < SLOTS) add_slot(no, ns, (unsigned)(w - base));
                else no |= SLOW_MARK;
            }
            if (full || x > x0) fin |= 1u << (8 * k);
            if (full || y > y0) fout |= 1u << (8 * k);
        }
        if (v < TT) {
            s_in[v] = x;
            s_out[v] = y;
            s_nin[v] = ni;
            s_nout[v] = no;
        }
    }
    {
        // honest roofline accounting: only visited tiles move bytes (SURVEY 8(d) terms)
        (void)me;                                 // = optr[base + cnt] - optr[base], one atomic per visit
        if (tid == 0) {
            atomicAdd(&dc->visit_e, (unsigned long long)(__ldg(g.optr + base + cnt) - __ldg(g.optr + base)));
            atomicAdd(&dc->visit_v, (unsigned long long)cnt);
        }
    }
    if (tid == 0) PROF_ADD(dc, 0, 1);                         // tile visits
    // ---- step 1b: recompute flags (pull model).  Byte k of s_fin[t] / s_fout[t] asks
    // vertex 4t+k to re-pull v_in / v_out from its intra-tile neighbours.  First visit:
    // everybody; otherwise the intra-tile dependents of what step 1 raised.
    s_fin[tid] = full ? 0x01010101u : 0u;
    s_fout[tid] = full ? 0x01010101u : 0u;
    __syncthreads();
    if (!full && (fin | fout)) {
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            const int v = tid * VPT + k;
            if ((fin >> (8 * k)) & 0xFF) notify(s_nout[v], g.optr, g.oadj, base, cnt, v, (uint8_t*)s_fin);
            if ((fout >> (8 * k)) & 0xFF) notify(s_nin[v], g.iptr, g.iadj, base, cnt, v, (uint8_t*)s_fout);
        }
    }
    __syncthreads();
#ifdef ECL_PROF
    const long long t_step1 = clock64();
    unsigned prof_rounds = 0, prof_drains = 0, prof_pushes = 0;
#endif
    // ---- step 2: local fixed point in shared memory, owner-computes pull (Alg. 1
    // l.10-11 on intra-tile edges).  A flagged vertex re-pulls the max over its intra
    // neighbours (slots, or its global row when it has more than SLOTS of them); if it
    // rises it stores the value (single writer) and flags its dependents with plain byte
    // stores after a block fence.  A thread takes its flag words with an exchange (only
    // when non-zero), which orders it after every setter it consumed.  Flagged items of a
    // warp are compacted into a per-warp queue so all lanes run the same path; each warp
    // drains its own 128 vertices, block rounds repeat until a round does no work.  No
    // shared-memory atomic touches the signatures.
    if (!SYNC) {
#ifndef ECL_PROF
        unsigned prof_rounds = 0, prof_drains = 0, prof_pushes = 0;
#endif
        drain_local(g, s_in, s_out, s_nin, s_nout, s_fin, s_fout, s_queue, base, cnt, prof_rounds, prof_drains,
                    prof_pushes);
    }
#ifdef ECL_PROF
    __syncthreads();
    const long long t_step2 = clock64();
    prof_pushes = warp_sum(prof_pushes);
    if ((tid & 31) == 0) { PROF_ADD(dc, 2, prof_drains); PROF_ADD(dc, 3, prof_pushes); }
    if (tid == 0) PROF_ADD(dc, 1, prof_rounds);
#endif
    // ---- step 3: write back; a raised v_in must reach the out-neighbours' tiles, a
    // raised v_out the in-neighbours' tiles (next pass).  Only this tile writes its
    // vertices, so global memory still holds the values read in step 1.
    int ch = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int v = tid * VPT + k;
        if (v >= cnt) continue;
        const int gi = base + v;
        const int x = s_in[v], y = s_out[v];
        if (x > ld_cg(cin + gi)) {
            cin[gi] = x;
            ch = 1;
            if (mark.on())
                for (int e = __ldg(g.optr + gi), ee = __ldg(g.optr + gi + 1); e < ee; e++) {
                    const int w = __ldg(g.oadj + e);
                    if ((unsigned)(w - base) >= (unsigned)cnt) mark(w / TT);
                }
        }
        if (y > ld_cg(cout + gi)) {
            cout[gi] = y;
            ch = 1;
            if (mark.on())
                for (int e = __ldg(g.iptr + gi), ee = __ldg(g.iptr + gi + 1); e < ee; e++) {
                    const int u = __ldg(g.iadj + e);
                    if ((unsigned)(u - base) >= (unsigned)cnt) mark(u / TT);
                }
        }
    }
    const int any_ch = __syncthreads_or(ch);
#ifdef ECL_PROF
    if (tid == 0) {
        const long long t_end = clock64();
        PROF_ADD(dc, 4, t_step1 - t_start);
        PROF_ADD(dc, 5, t_step2 - t_step1);
        PROF_ADD(dc, 6, t_end - t_step2);
    }
#endif
    return any_ch;
}

template <bool SYNC, int TT>
static __global__ void __launch_bounds__(TT / VPT, (1536 / (TT / VPT)) > 0 ? 1536 / (TT / VPT) : 1)
k_prop_tile(WGraph g, int32_t* __restrict__ cin, int32_t* __restrict__ cout, DevCounters* __restrict__ dc, int pass,
            int first, uint8_t* __restrict__ dirty_cur, uint8_t* __restrict__ dirty_next, int full, int run) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ unsigned s_fin[TT / VPT], s_fout[TT / VPT];             // raise flags, byte k = vertex 4t+k
    __shared__ unsigned short s_queue[2 * TT];                         // per-warp item queues
    __shared__ int s_dirty;
    TileSmem<TT> S;
    S.s_in = (int*)smem_raw;
    S.s_out = S.s_in + TT;
    S.s_nin = (unsigned long long*)(S.s_out + TT);
    S.s_nout = S.s_nin + TT;
    S.s_fin = s_fin;
    S.s_fout = s_fout;
    S.s_queue = s_queue;
    if (!pass_begin(dc, pass, first)) return;
    const int ntiles = (g.na + TT - 1) / TT;
    const int tid = threadIdx.x;
    int ch_any = 0;
    // Each CTA walks a run of `run` consecutive tiles in order (reversed on odd passes):
    // a tile then sees the tile before it in the run already finished (Gauss-Seidel along
    // the run), while different runs proceed in parallel.
    for (int j = 0; j < run; j++) {
        const int idx = (int)blockIdx.x * run + ((pass & 1) ? run - 1 - j : j);
        if (idx >= ntiles) continue;
        const int tile = (pass & 1) ? ntiles - 1 - idx : idx;
        // dirty-tile skipping: a tile whose inputs did not change since its last visit is
        // at its local fixed point already.  The read flag is cleared here, so after pass p
        // the buffer read in pass p is all zero and pass p+1 can fill it for pass p+2.
        if (dirty_cur) {
            if (tid == 0) {
                s_dirty = dirty_cur[tile];
                dirty_cur[tile] = 0;
            }
            __syncthreads();
            const int d = s_dirty;
            __syncthreads();             // everyone has read s_dirty before thread 0 rewrites it
            if (!d) continue;
        }
        ch_any |= tile_visit<SYNC, TT>(g, cin, cout, dc, tile, full, MarkNext{dirty_next}, S);
        __syncthreads();                                     // shared memory is reused by the next tile
    }
    if (ch_any && tid == 0) dc->changed[pass & (RING - 1)] = 1;
}

}  // namespace eclscc
