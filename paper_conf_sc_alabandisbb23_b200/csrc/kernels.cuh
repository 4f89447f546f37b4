// kernels.cuh -- sm_100a kernels of the ECL-SCC hot path.
//
// Citation key: P:n = PAPER.md line n.  Steps:
//   a1 k_validate, k_indeg, k_csc_scatter       CSR -> CSC transpose of the input
//   a2/a7 k_keep_count, k_compact_count, k_compact_scatter
//                                               Phase 3 edge removal
//                                               fused with one Trim-1 round and the
//                                               compaction of CSR and CSC
//   a3 k_reset                                  Phase 1 for the next iteration
//   a4-a6 k_prop                                Phase 2 max propagation
#pragma once
#include "common.cuh"

namespace eclscc {

// ------------------------------------------------------------------ init / validation
__global__ void k_init_sig(int32_t n, int32_t* __restrict__ vin, int32_t* __restrict__ vout) {
    // Alg. 1 l.3-6: v_in <- v_id, v_out <- v_id
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        vin[v] = (int32_t)v;
        vout[v] = (int32_t)v;
    }
}

__global__ void k_validate(int32_t n, int64_t nnz, const int32_t* __restrict__ rp,
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
__global__ void k_indeg(int64_t nnz, const int32_t* __restrict__ ci, int32_t* __restrict__ ideg) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&ideg[ci[e]], 1);
}

// one thread per source row; rows longer than HEAVY are spread over the warp
__global__ void k_csc_scatter(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                              const int32_t* __restrict__ iptr, int32_t* __restrict__ cursor,
                              int32_t* __restrict__ iadj) {
    const int lane = threadIdx.x & 31;
    const int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool valid = u < n;
    int b = 0, e = 0;
    if (valid) { b = rp[u]; e = rp[u + 1]; }
    if (valid && e - b <= HEAVY)
        for (int k = b; k < e; k++) {
            const int w = ci[k];
            iadj[iptr[w] + atomicAdd(&cursor[w], 1)] = (int32_t)u;
        }
    unsigned hm = __ballot_sync(FULL, valid && e - b > HEAVY);
    while (hm) {
        const int src = __ffs(hm) - 1;
        hm &= hm - 1;
        const int sb = __shfl_sync(FULL, b, src), se = __shfl_sync(FULL, e, src);
        const int su = __shfl_sync(FULL, (int)u, src);
        for (int k = sb + lane; k < se; k += WARP) {
            const int w = ci[k];
            iadj[iptr[w] + atomicAdd(&cursor[w], 1)] = su;
        }
    }
}

// ------------------------------------------------------------------ Phase 3 predicates
// keep(u->w) in iteration k >= 2 (P:147 negated): both endpoints carry the same
// (in, out) pair and that pair is unfinished (in != out).  Evaluated from either end: the
// row owner's pair (a, b) is passed in, the other endpoint's pair is gathered.
// In the first removal (FIRST) every edge except a self-loop is kept (DESIGN reading 9).
template <bool FIRST>
__device__ __forceinline__ bool keep_edge(int owner, int a, int other, const int32_t* __restrict__ vin,
                                          const int32_t* __restrict__ vout, int b) {
    if (FIRST) return other != owner;
    return ld_cg(vin + other) == a && ld_cg(vout + other) == b;
}
// Trim-1 on the kept graph: a vertex without a kept in-edge or out-edge
__device__ __forceinline__ bool trimmed(const int32_t* __restrict__ kin, const int32_t* __restrict__ kout, int x) {
    return ld_cg(kin + x) == 0 || ld_cg(kout + x) == 0;
}

struct RowCtx {
    int v, ob, oe, ib, ie, a, b;
    bool valid, live;
};

template <bool FIRST>
__device__ __forceinline__ RowCtx load_row(const WGraph& g, int64_t i, const int32_t* __restrict__ vin,
                                           const int32_t* __restrict__ vout) {
    RowCtx r{};
    r.valid = i < g.na;
    if (r.valid) {
        r.v = g.act ? g.act[i] : (int)i;
        r.ob = g.optr[i]; r.oe = g.optr[i + 1];
        r.ib = g.iptr[i]; r.ie = g.iptr[i + 1];
        if (!FIRST) { r.a = ld_cg(vin + r.v); r.b = ld_cg(vout + r.v); }
    }
    r.live = r.valid && (FIRST || r.a != r.b);
    return r;
}

// kept in/out degree per vertex (global-indexed), plus the number of kept edges
template <bool FIRST>
__global__ void k_keep_count(WGraph g, const int32_t* __restrict__ vin, const int32_t* __restrict__ vout,
                             int32_t* __restrict__ kin, int32_t* __restrict__ kout,
                             unsigned long long* __restrict__ kept) {
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const RowCtx r = load_row<FIRST>(g, i, vin, vout);
    int co = 0, ci = 0;
    if (r.live && r.oe - r.ob <= HEAVY)
        for (int e = r.ob; e < r.oe; e++) co += keep_edge<FIRST>(r.v, r.a, g.oadj[e], vin, vout, r.b);
    if (r.live && r.ie - r.ib <= HEAVY)
        for (int e = r.ib; e < r.ie; e++) ci += keep_edge<FIRST>(r.v, r.a, g.iadj[e], vin, vout, r.b);
    for (int dir = 0; dir < 2; dir++) {
        const int rb = dir ? r.ib : r.ob, re = dir ? r.ie : r.oe;
        const int32_t* adj = dir ? g.iadj : g.oadj;
        unsigned hm = __ballot_sync(FULL, r.live && re - rb > HEAVY);
        while (hm) {
            const int src = __ffs(hm) - 1;
            hm &= hm - 1;
            const int sb = __shfl_sync(FULL, rb, src), se = __shfl_sync(FULL, re, src);
            const int sv = __shfl_sync(FULL, r.v, src), sa = __shfl_sync(FULL, r.a, src);
            const int sbb = __shfl_sync(FULL, r.b, src);
            int c = 0;
            for (int e = sb + lane; e < se; e += WARP) c += keep_edge<FIRST>(sv, sa, adj[e], vin, vout, sbb);
            c = warp_sum(c);
            if (lane == src) { if (dir) ci = c; else co = c; }
        }
    }
    if (r.valid) { kin[r.v] = ci; kout[r.v] = co; }
    const int s = warp_sum(co);
    if (lane == 0 && s) atomicAdd(kept, (unsigned long long)s);
}

// surviving (kept and not trimmed) degree of one row; light rows by the lane, heavy rows
// by the warp
template <bool FIRST, bool TRIM>
__device__ __forceinline__ void survivor_counts(const WGraph& g, const RowCtx& r, bool vtrim,
                                                const int32_t* __restrict__ vin, const int32_t* __restrict__ vout,
                                                const int32_t* __restrict__ kin, const int32_t* __restrict__ kout,
                                                int lane, int& nout, int& nin) {
    nout = 0; nin = 0;
    const bool go = r.live && !vtrim;
    if (!TRIM) {
        if (go) { nout = ld_cg(kout + r.v); nin = ld_cg(kin + r.v); }
        return;
    }
    if (go && r.oe - r.ob <= HEAVY)
        for (int e = r.ob; e < r.oe; e++) {
            const int w = g.oadj[e];
            nout += keep_edge<FIRST>(r.v, r.a, w, vin, vout, r.b) && !trimmed(kin, kout, w);
        }
    if (go && r.ie - r.ib <= HEAVY)
        for (int e = r.ib; e < r.ie; e++) {
            const int u = g.iadj[e];
            nin += keep_edge<FIRST>(r.v, r.a, u, vin, vout, r.b) && !trimmed(kin, kout, u);
        }
    for (int dir = 0; dir < 2; dir++) {
        const int rb = dir ? r.ib : r.ob, re = dir ? r.ie : r.oe;
        const int32_t* adj = dir ? g.iadj : g.oadj;
        unsigned hm = __ballot_sync(FULL, go && re - rb > HEAVY);
        while (hm) {
            const int src = __ffs(hm) - 1;
            hm &= hm - 1;
            const int sb = __shfl_sync(FULL, rb, src), se = __shfl_sync(FULL, re, src);
            const int sv = __shfl_sync(FULL, r.v, src), sa = __shfl_sync(FULL, r.a, src);
            const int sbb = __shfl_sync(FULL, r.b, src);
            int c = 0;
            for (int e = sb + lane; e < se; e += WARP) {
                const int x = adj[e];
                c += keep_edge<FIRST>(sv, sa, x, vin, vout, sbb) && !trimmed(kin, kout, x);
            }
            c = warp_sum(c);
            if (lane == src) { if (dir) nin = c; else nout = c; }
        }
    }
}

// per-warp totals (alive vertices, surviving out-edges, surviving in-edges)
template <bool FIRST, bool TRIM>
__global__ void k_compact_count(WGraph g, const int32_t* __restrict__ vin, const int32_t* __restrict__ vout,
                                const int32_t* __restrict__ kin, const int32_t* __restrict__ kout,
                                int4* __restrict__ wsum) {
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const RowCtx r = load_row<FIRST>(g, i, vin, vout);
    const bool vtrim = TRIM && r.live && trimmed(kin, kout, r.v);
    int nout, nin;
    survivor_counts<FIRST, TRIM>(g, r, vtrim, vin, vout, kin, kout, lane, nout, nin);
    const int alive = (nout + nin) > 0;
    const int sa = warp_sum(alive), so = warp_sum(nout), si = warp_sum(nin);
    if (lane == 0) wsum[i >> 5] = make_int4(sa, so, si, 0);
}

// write one row's survivors starting at dst[pos]; light rows by the lane, heavy by the warp
template <bool FIRST, bool TRIM>
__device__ __forceinline__ void emit_rows(const int32_t* __restrict__ adj, int rb, int re, bool go, int pos,
                                          const RowCtx& r, const int32_t* __restrict__ vin,
                                          const int32_t* __restrict__ vout, const int32_t* __restrict__ kin,
                                          const int32_t* __restrict__ kout, int32_t* __restrict__ dst, int lane) {
    if (go && re - rb <= HEAVY) {
        for (int e = rb; e < re; e++) {
            const int x = adj[e];
            if (keep_edge<FIRST>(r.v, r.a, x, vin, vout, r.b) && !(TRIM && trimmed(kin, kout, x))) dst[pos++] = x;
        }
    }
    unsigned hm = __ballot_sync(FULL, go && re - rb > HEAVY);
    while (hm) {
        const int src = __ffs(hm) - 1;
        hm &= hm - 1;
        const int sb = __shfl_sync(FULL, rb, src), se = __shfl_sync(FULL, re, src);
        const int sv = __shfl_sync(FULL, r.v, src), sa = __shfl_sync(FULL, r.a, src);
        const int sbb = __shfl_sync(FULL, r.b, src);
        int spos = __shfl_sync(FULL, pos, src);
        for (int base = sb; base < se; base += WARP) {
            const int e = base + lane;
            bool k = false;
            int x = 0;
            if (e < se) {
                x = adj[e];
                k = keep_edge<FIRST>(sv, sa, x, vin, vout, sbb) && !(TRIM && trimmed(kin, kout, x));
            }
            const unsigned bm = __ballot_sync(FULL, k);
            if (k) dst[spos + __popc(bm & ((1u << lane) - 1))] = x;
            spos += __popc(bm);
        }
    }
}

// stable compaction: new active list, new CSR/CSC offsets and adjacency
template <bool FIRST, bool TRIM>
__global__ void k_compact_scatter(WGraph g, const int32_t* __restrict__ vin, const int32_t* __restrict__ vout,
                                  const int32_t* __restrict__ kin, const int32_t* __restrict__ kout,
                                  const int4* __restrict__ wscan, const int4* __restrict__ totals,
                                  int32_t* __restrict__ act2, int32_t* __restrict__ optr2, int32_t* __restrict__ oadj2,
                                  int32_t* __restrict__ iptr2, int32_t* __restrict__ iadj2) {
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i == 0) {
        const int4 t = *totals;
        optr2[t.x] = t.y;
        iptr2[t.x] = t.z;
    }
    const RowCtx r = load_row<FIRST>(g, i, vin, vout);
    const bool vtrim = TRIM && r.live && trimmed(kin, kout, r.v);
    int nout, nin;
    survivor_counts<FIRST, TRIM>(g, r, vtrim, vin, vout, kin, kout, lane, nout, nin);
    const int alive = (nout + nin) > 0;
    const int4 base = wscan[i >> 5];
    const int pa = warp_incl_scan(alive, lane) - alive + base.x;
    const int po = warp_incl_scan(nout, lane) - nout + base.y;
    const int pi = warp_incl_scan(nin, lane) - nin + base.z;
    if (alive) {
        act2[pa] = r.v;
        optr2[pa] = po;
        iptr2[pa] = pi;
    }
    const bool go = r.live && !vtrim;
    emit_rows<FIRST, TRIM>(g.oadj, r.ob, r.oe, go, po, r, vin, vout, kin, kout, oadj2, lane);
    emit_rows<FIRST, TRIM>(g.iadj, r.ib, r.ie, go, pi, r, vin, vout, kin, kout, iadj2, lane);
}

// Phase 1 of the next iteration (R2, DESIGN reading 1): unfinished vertices restart from
// their own ID; this also finalises vertices that just lost their last edge.
__global__ void k_reset(WGraph g, int32_t* __restrict__ vin, int32_t* __restrict__ vout) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= g.na) return;
    const int v = g.act ? g.act[i] : (int)i;
    if (vin[v] != vout[v]) { vin[v] = v; vout[v] = v; }
}

// ------------------------------------------------------------------ Phase 2
// One global relaxation pass (Alg. 1 l.9-11), pull form: the owner of v gathers
//   in[v]  <- max(in[v],  in[u])   over live in-edges  u->v   (l.11)
//   out[v] <- max(out[v], out[w])  over live out-edges v->w   (l.10)
// With COMPRESS the gathered value is in[in[u]] / out[out[w]].  Values are
// written in place (owner writes, so no atomics); concurrent readers see the old or the
// new value, both valid ancestors/descendants (monotone).  A pass that changes
// nothing observed a consistent snapshot, so it certifies the fixed point.
//
// Pass protocol: pass p clears changed[p+1]; it returns at once if pass p-1 changed
// nothing; otherwise it sets changed[p] if it wrote anything.
template <bool COMPRESS>
__global__ void __launch_bounds__(256) k_prop(WGraph g, int32_t* __restrict__ vin, int32_t* __restrict__ vout,
                                              DevCounters* __restrict__ dc, int pass) {
    // every pass (also a skipped one) clears its successor's word, so changed[p] is 0
    // unless pass p itself ran and changed something
    if (blockIdx.x == 0 && threadIdx.x == 0) dc->changed[(pass + 1) & (RING - 1)] = 0;
    if (pass > 0 && ld_vol(&dc->changed[(pass - 1) & (RING - 1)]) == 0) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(&dc->passes, 1ull);
    const int lane = threadIdx.x & 31;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool valid = i < g.na;
    int v = 0, ob = 0, oe = 0, ib = 0, ie = 0, x0 = 0, y0 = 0;
    if (valid) {
        v = g.act ? g.act[i] : (int)i;
        ob = g.optr[i]; oe = g.optr[i + 1];
        ib = g.iptr[i]; ie = g.iptr[i + 1];
        x0 = ld_cg(vin + v);
        y0 = ld_cg(vout + v);
    }
    int x = x0, y = y0;
    if (valid && ie - ib <= HEAVY)
        for (int e = ib; e < ie; e++) {
            int t = ld_cg(vin + g.iadj[e]);
            if (COMPRESS) t = ld_cg(vin + t);
            x = max(x, t);
        }
    if (valid && oe - ob <= HEAVY)
        for (int e = ob; e < oe; e++) {
            int t = ld_cg(vout + g.oadj[e]);
            if (COMPRESS) t = ld_cg(vout + t);
            y = max(y, t);
        }
    {
        unsigned hm = __ballot_sync(FULL, valid && ie - ib > HEAVY);
        while (hm) {
            const int src = __ffs(hm) - 1;
            hm &= hm - 1;
            const int sb = __shfl_sync(FULL, ib, src), se = __shfl_sync(FULL, ie, src);
            int acc = 0;
            for (int e = sb + lane; e < se; e += WARP) {
                int t = ld_cg(vin + g.iadj[e]);
                if (COMPRESS) t = ld_cg(vin + t);
                acc = max(acc, t);
            }
            acc = warp_max(acc);
            if (lane == src) x = max(x, acc);
        }
        hm = __ballot_sync(FULL, valid && oe - ob > HEAVY);
        while (hm) {
            const int src = __ffs(hm) - 1;
            hm &= hm - 1;
            const int sb = __shfl_sync(FULL, ob, src), se = __shfl_sync(FULL, oe, src);
            int acc = 0;
            for (int e = sb + lane; e < se; e += WARP) {
                int t = ld_cg(vout + g.oadj[e]);
                if (COMPRESS) t = ld_cg(vout + t);
                acc = max(acc, t);
            }
            acc = warp_max(acc);
            if (lane == src) y = max(y, acc);
        }
    }
    bool ch = false;
    if (x > x0) { vin[v] = x; ch = true; }
    if (y > y0) { vout[v] = y; ch = true; }
    if (__any_sync(FULL, ch) && lane == 0) dc->changed[pass & (RING - 1)] = 1;
}

}  // namespace eclscc
