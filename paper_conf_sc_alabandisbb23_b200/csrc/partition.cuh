// partition.cuh -- kernels of the edge-partitioned (multi-GPU) mode.
//
// A rank owns the out-edges of source rows [rb, re) (global destination IDs) and the
// transpose of exactly those edges (a CSC over all n vertices).  Signatures v_in / v_out
// are REPLICATED: global-indexed arrays of n entries on every rank, combined with an
// all-reduce(MAX) after every local fixed point.  Edge removal (P:145-153,
// P:186) is local: each rank filters its own edges with the same predicate on identical
// replicas.  Rows are compacted in place (row starts fixed, live degree per row).
#pragma once
#include "common.cuh"

namespace eclscc {
namespace part {

// ------------------------------------------------------------------ ingest
static __global__ void k_validate_part(int32_t nrows, int64_t nnz, const int32_t* __restrict__ rp,
                                const int32_t* __restrict__ ci, int32_t ncols, int* __restrict__ err) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int bad = 0;
    for (int64_t v = t0; v < nrows; v += stride) {
        const int32_t a = rp[v], b = rp[v + 1];
        if (a > b) bad = 1;
        if (v == 0 && a != 0) bad = 1;
        if (v == nrows - 1 && (int64_t)b != nnz) bad = 1;
    }
    for (int64_t e = t0; e < nnz; e += stride) {
        const int32_t c = ci[e];
        if (c < 0 || c >= ncols) bad = 1;
    }
    if (bad) *err = 1;
}

// working CSR copy (self-loops dropped, DESIGN reading 9) and the live out-degree
static __global__ void k_copy_rows(int32_t nrows, int32_t rb, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                            int32_t* __restrict__ wci, int32_t* __restrict__ odeg) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    const int u = rb + (int)r;
    int k = rp[r];
    for (int e = rp[r]; e < rp[r + 1]; e++) {
        const int w = ci[e];
        if (w != u) wci[k++] = w;
    }
    odeg[r] = k - rp[r];
}
static __global__ void k_indeg_rows(int32_t nrows, const int32_t* __restrict__ rp, const int32_t* __restrict__ wci,
                             const int32_t* __restrict__ odeg, int32_t* __restrict__ ideg) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    for (int e = rp[r]; e < rp[r] + odeg[r]; e++) atomicAdd(&ideg[wci[e]], 1);
}
static __global__ void k_csc_rows(int32_t nrows, int32_t rb, const int32_t* __restrict__ rp, const int32_t* __restrict__ wci,
                           const int32_t* __restrict__ odeg, const int32_t* __restrict__ cp, int32_t* __restrict__ cursor,
                           int32_t* __restrict__ cr) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    for (int e = rp[r]; e < rp[r] + odeg[r]; e++) {
        const int w = wci[e];
        cr[cp[w] + atomicAdd(&cursor[w], 1)] = rb + (int)r;
    }
}

// ------------------------------------------------------------------ Phase 2 (local)
// One relaxation pass over this rank's edges (Alg. 1 l.9-11, pull): out-rows of the
// owned sources, in-columns of every destination.  Owner-writes in place.  Ring protocol
// as in kernels.cuh: the rows kernel (first of the pass) clears ring[p+1]; both return
// at once if pass p-1 changed nothing; a raise sets ring[p].
// Local Phase-2 passes with block-local iteration ("every thread block internally
// iterates until none of the edges assigned to it propagate any more values"): a CTA owns
// PART_RPT x blockDim consecutive rows (columns) and repeats its pulls until a block round
// raises nothing, so chains inside its range converge in one launch instead of one launch
// per hop.  Other CTAs' values are read through L2 (ld.cg); the ring word of the pass is set
// if anything rose (the driver repeats passes until one raises nothing: a fixed point).
// `touched` is set by every pass that raised a value and is reset only when the rank's
// local phase starts: the ring words are recycled every RING passes, so a rank whose local
// fixed point took a multiple of RING passes would otherwise report "no change".
constexpr int PART_RPT = 4;
static __global__ void __launch_bounds__(256) k_prop_rows(int32_t nrows, int32_t rb, const int32_t* __restrict__ rp,
                                                          const int32_t* __restrict__ wci, const int32_t* __restrict__ odeg,
                                                          int32_t* __restrict__ vout, int* __restrict__ ring, int pass,
                                                          int* __restrict__ touched) {
    if (blockIdx.x == 0 && threadIdx.x == 0) ring[(pass + 1) & (RING - 1)] = 0;
    if (pass > 0 && ld_vol(ring + ((pass - 1) & (RING - 1))) == 0) return;
    const int64_t r0 = (int64_t)blockIdx.x * blockDim.x * PART_RPT + threadIdx.x;
    int any = 0;
    for (;;) {
        int ch = 0;
#pragma unroll
        for (int k = 0; k < PART_RPT; k++) {
            const int64_t r = r0 + (int64_t)k * blockDim.x;
            if (r >= nrows) break;
            const int u = rb + (int)r;
            const int y0 = ld_cg(vout + u);
            int y = y0;
            for (int e = rp[r], ee = rp[r] + odeg[r]; e < ee; e++) y = max(y, ld_cg(vout + wci[e]));
            if (y > y0) { __stcg(vout + u, y); ch = 1; }
        }
        if (!__syncthreads_or(ch)) break;
        any = 1;
    }
    if (any && threadIdx.x == 0) {
        ring[pass & (RING - 1)] = 1;
        *touched = 1;                 // never cleared by the ring protocol (see multi.cu)
    }
}
static __global__ void __launch_bounds__(256) k_prop_cols(int32_t n, const int32_t* __restrict__ cp, const int32_t* __restrict__ cr,
                                                          const int32_t* __restrict__ ideg, int32_t* __restrict__ vin,
                                                          int* __restrict__ ring, int pass, int* __restrict__ touched) {
    if (pass > 0 && ld_vol(ring + ((pass - 1) & (RING - 1))) == 0) return;
    const int64_t w0 = (int64_t)blockIdx.x * blockDim.x * PART_RPT + threadIdx.x;
    int any = 0;
    for (;;) {
        int ch = 0;
#pragma unroll
        for (int k = 0; k < PART_RPT; k++) {
            const int64_t w = w0 + (int64_t)k * blockDim.x;
            if (w >= n) break;
            if (ideg[w] == 0) continue;
            const int x0 = ld_cg(vin + w);
            int x = x0;
            for (int e = cp[w], ee = cp[w] + ideg[w]; e < ee; e++) x = max(x, ld_cg(vin + cr[e]));
            if (x > x0) { __stcg(vin + w, x); ch = 1; }
        }
        if (!__syncthreads_or(ch)) break;
        any = 1;
    }
    if (any && threadIdx.x == 0) {
        ring[pass & (RING - 1)] = 1;
        *touched = 1;                 // never cleared by the ring protocol (see multi.cu)
    }
}

// ------------------------------------------------------------------ Phase 3 + trim
// keep u->w iff (in,out)(u) == (in,out)(w) and in(u) != out(u); rows and
// columns filtered in place with the same predicate.  first: keep every edge (the input
// minus self-loops, already dropped).  Writes kept degrees into kout (rows, by global ID)
// and kin (columns, partial per rank: summed over ranks afterwards).
__device__ __forceinline__ bool keep_pair(const int32_t* vin, const int32_t* vout, int u, int w) {
    const int a = vin[u], b = vout[u];
    return a != b && vin[w] == a && vout[w] == b;
}
static __global__ void k_keep_rows(int32_t nrows, int32_t rb, const int32_t* __restrict__ rp, int32_t* __restrict__ wci,
                            int32_t* __restrict__ odeg, const int32_t* __restrict__ vin, const int32_t* __restrict__ vout,
                            int first, int32_t* __restrict__ kout) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    const int u = rb + (int)r;
    int k = rp[r];
    for (int e = rp[r]; e < rp[r] + odeg[r]; e++) {
        const int w = wci[e];
        if (first || keep_pair(vin, vout, u, w)) wci[k++] = w;
    }
    odeg[r] = k - rp[r];
    kout[u] = k - rp[r];
}
static __global__ void k_keep_cols(int32_t n, const int32_t* __restrict__ cp, int32_t* __restrict__ cr, int32_t* __restrict__ ideg,
                            const int32_t* __restrict__ vin, const int32_t* __restrict__ vout, int first,
                            int32_t* __restrict__ kin) {
    const int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (w >= n) return;
    int k = cp[w];
    for (int e = cp[w]; e < cp[w] + ideg[w]; e++) {
        const int u = cr[e];
        if (first || keep_pair(vin, vout, u, (int)w)) cr[k++] = u;
    }
    ideg[w] = k - cp[w];
    kin[w] = k - cp[w];
}
// Trim-1 with GLOBAL kept degrees (kin/kout all-reduced): drop edges at trimmed
// endpoints; count surviving edges of this rank.
__device__ __forceinline__ bool trimmed_g(const int32_t* kin, const int32_t* kout, int x) {
    return kin[x] == 0 || kout[x] == 0;
}
static __global__ void k_trim_rows(int32_t nrows, int32_t rb, const int32_t* __restrict__ rp, int32_t* __restrict__ wci,
                            int32_t* __restrict__ odeg, const int32_t* __restrict__ kin, const int32_t* __restrict__ kout,
                            int trim, unsigned long long* __restrict__ live) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int cnt = 0;
    if (r < nrows) {
        const int u = rb + (int)r;
        int k = rp[r];
        const bool tu = trim && trimmed_g(kin, kout, u);
        for (int e = rp[r]; e < rp[r] + odeg[r]; e++) {
            const int w = wci[e];
            if (!tu && !(trim && trimmed_g(kin, kout, w))) wci[k++] = w;
        }
        odeg[r] = k - rp[r];
        cnt = k - rp[r];
    }
    cnt = warp_sum(cnt);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(live, (unsigned long long)cnt);
}
static __global__ void k_trim_cols(int32_t n, const int32_t* __restrict__ cp, int32_t* __restrict__ cr, int32_t* __restrict__ ideg,
                            const int32_t* __restrict__ kin, const int32_t* __restrict__ kout, int trim) {
    const int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (w >= n) return;
    int k = cp[w];
    const bool tw = trim && trimmed_g(kin, kout, (int)w);
    for (int e = cp[w]; e < cp[w] + ideg[w]; e++) {
        const int u = cr[e];
        if (!tw && !(trim && trimmed_g(kin, kout, u))) cr[k++] = u;
    }
    ideg[w] = k - cp[w];
}
// Phase 1 on the replica (R2): unfinished vertices restart from pi(v)
static __global__ void k_reset_all(int32_t n, int32_t* __restrict__ vin, int32_t* __restrict__ vout, Prio P) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        if (vin[v] != vout[v]) {
            const int pv = (int)prio_of(P, (uint32_t)v);
            vin[v] = pv;
            vout[v] = pv;
        }
}
static __global__ void k_init_prio(int32_t n, int32_t* __restrict__ vin, int32_t* __restrict__ vout, Prio P) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int pv = (int)prio_of(P, (uint32_t)v);
        vin[v] = pv;
        vout[v] = pv;
    }
}
// labels: every signature is final (in == out); encode -(s+1) for k_relabel_* (or the
// raw ID label itself with identity priorities)
static __global__ void k_encode_labels(int32_t n, const int32_t* __restrict__ vin, int32_t* __restrict__ labels, int ids) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        labels[v] = ids ? vin[v] : -(vin[v] + 1);
}
// emulated all-reduce over P replicas on one device: MAX (op 0) or SUM (op 1)
static __global__ void k_reduce_replicas(int P, int32_t* const* __restrict__ bufs, int64_t count, int op) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        int acc = bufs[0][i];
        for (int r = 1; r < P; r++) acc = op == 0 ? max(acc, bufs[r][i]) : acc + bufs[r][i];
        for (int r = 0; r < P; r++) bufs[r][i] = acc;
    }
}

}  // namespace part
}  // namespace eclscc
