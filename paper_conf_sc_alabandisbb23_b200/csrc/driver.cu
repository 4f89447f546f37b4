// driver.cu -- plan/workspace, the outer loop of Alg. 1, and the C ABI (include/ecl_scc.h).
//
// Outer loop (Alg. 1 l.2-21) as run here, rule R2 (reading 1):
//   ingest:  v_in = v_out = v (l.3-6); CSC transpose of the input CSR
//   repeat:  edge removal + Trim-1 + compaction  (Phase 3 of the previous iteration,
//            l.15-19 and P:186), then Phase 1 for the unfinished (l.3-6),
//            stop if no live edge is left (reading 2), else
//            Phase 2 to its fixed point (l.7-14).
// labels_out doubles as the v_in array, so the final signatures need no copy.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "../../include/ecl_scc.h"
#include "common.cuh"
#include "kernels.cuh"
#include "scan.cuh"
#include "reorder.cuh"
#include "pack.cuh"
#include "cluster.cuh"
#include "levels.cuh"
#include "partition.cuh"
#include "driver.h"

namespace eclscc {

static thread_local char g_err[512] = "";

int fail(int status, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return status;
}
void clear_err() { g_err[0] = 0; }
const char* last_err() { return g_err; }

#define CK(call)                                                                                      \
    do {                                                                                              \
        cudaError_t _e = (call);                                                                      \
        if (_e != cudaSuccess)                                                                        \
            return fail(ECL_SCC_ECUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(_e)); \
    } while (0)

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
static inline unsigned grid_for(int64_t work, int threads) {
    int64_t g = cdiv(work, threads);
    if (g < 1) g = 1;
    return (unsigned)std::min<int64_t>(g, 0x7FFFFFFF);
}

constexpr int TPB = 256;
static_assert(TPB == TPB_COMPACT, "k_keep_count reduces over TPB_COMPACT threads");
constexpr double REORDER_LOCALITY = 0.85;   // measured: C4 lex 0.77, blocked8 0.91
// the reordering's cost is mostly per BFS level (launches, host checks): below this size it
// does not pay back (measured: C2 lex, 1M vertices, 2.98 ms without vs 3.95 ms with)
constexpr int32_t REORDER_MIN_N = 1 << 22;
// a block-local fixed point pays only if tiles hold a real share of the edges (measured:
// C3, random IDs, ~0 local edges: 8.2 ms with plain Jacobi passes vs 9.3 ms)
constexpr double LOCAL_FP_LOCALITY = 0.25;

// --------------------------------------------------------------------------- plan
int plan_alloc(Plan* p, int32_t n_max, int64_t m_max) {
    p->n_cap = std::max<int32_t>(n_max, 1);
    p->m_cap = std::max<int64_t>(m_max, 1);
    const size_t n1 = (size_t)p->n_cap + 1;
    const size_t m = (size_t)p->m_cap;
    p->nw_cap = cdiv(p->n_cap, TPB) * (TPB / WARP) + 1;
    p->bsum_cap = cdiv(std::max<int64_t>(n1, p->nw_cap), SCAN_TILE) + 1;
    p->chunk_cap = 2 * (int64_t)m / HEAVY_T + 16;
    p->dirty_cap = cdiv(p->n_cap, 512) + 1;
    // development knobs, read once per plan; 0 = the measured default
    auto knob = [](const char* name, int lo, int hi) -> int {
        const char* e = getenv(name);
        return e ? std::min(hi, std::max(lo, atoi(e))) : 0;
    };
    p->knob_run = knob("ECL_SCC_RUN", 1, 64);
    p->knob_claim = knob("ECL_SCC_CLAIM", 1, 32);
    p->knob_claim_div = knob("ECL_SCC_CLAIM_DIV", 1, 64);
    p->knob_claim_max = knob("ECL_SCC_CLAIM_MAX", 1, 32);
    p->knob_async_ctas = knob("ECL_SCC_ASYNC_CTAS", 1, 8);
    p->knob_lv_ctas = knob("ECL_SCC_LV_CTAS", 1, 4096);
    p->lab_lo = 0;
    p->lab_hi = INT32_MAX;
    if (cudaGetDevice(&p->device) != cudaSuccess) {
        cudaGetLastError();
        return fail(ECL_SCC_ECUDA, "plan: no current CUDA device");
    }
    auto A = [&](void** ptr, size_t bytes) -> cudaError_t { return cudaMalloc(ptr, bytes); };
    cudaError_t e = cudaSuccess;
    for (int b = 0; b < 2; b++) {
        e = e ? e : A((void**)&p->act[b], n1 * 4);
        e = e ? e : A((void**)&p->cin[b], n1 * 4);
        e = e ? e : A((void**)&p->cout[b], n1 * 4);
        e = e ? e : A((void**)&p->optr[b], n1 * 4);
        e = e ? e : A((void**)&p->iptr[b], n1 * 4);
        e = e ? e : A((void**)&p->oadj[b], m * 4);
        e = e ? e : A((void**)&p->iadj[b], m * 4);
    }
    // one allocation, two views: the compaction's interleaved kept degrees kio[i] = {in, out}
    // (one 8-byte gather per far end in the trim), and two int arrays kin / kout of n+1 for
    // the ingest, the relabelling and the levels (never used at the same time)
    e = e ? e : A((void**)&p->kin, 2 * n1 * 4);
    if (e == cudaSuccess) {
        p->kout = p->kin + n1;
        p->kio = (int2*)p->kin;
    }
    if (p->flags & ECL_SCC_FOUR_SIG)
        for (int b = 0; b < 2; b++) {
            e = e ? e : A((void**)&p->min_in[b], n1 * 4);
            e = e ? e : A((void**)&p->min_out[b], n1 * 4);
        }
    if (p->flags & ECL_SCC_TRIM2) e = e ? e : A((void**)&p->t2, n1 * 4);
    if (p->flags & (ECL_SCC_COMPRESS | ECL_SCC_RAISE)) e = e ? e : A((void**)&p->slot, n1 * 4);
    e = e ? e : A((void**)&p->newidx, n1 * 4);
    e = e ? e : A((void**)&p->cnt, n1 * sizeof(int2));
    e = e ? e : A((void**)&p->emask, n1 * sizeof(uint2));
    e = e ? e : A((void**)&p->sig2, n1 * sizeof(int2));
    e = e ? e : A((void**)&p->wsum, (size_t)p->nw_cap * sizeof(int4));
    e = e ? e : A((void**)&p->wscan, (size_t)p->nw_cap * sizeof(int4));
    e = e ? e : A((void**)&p->bsum, (size_t)p->bsum_cap * sizeof(int4));
    e = e ? e : A((void**)&p->chunks, 2 * (size_t)p->chunk_cap * sizeof(Chunk));
    e = e ? e : A((void**)&p->chunk_cnt, (size_t)p->chunk_cap * sizeof(int));
    e = e ? e : A((void**)&p->hcnt, n1 * sizeof(int2));
    e = e ? e : A((void**)&p->dirty, 2 * (size_t)p->dirty_cap);
    e = e ? e : A((void**)&p->rp2, n1 * 4);
    e = e ? e : A((void**)&p->ci2, m * 4);
    e = e ? e : A((void**)&p->orig, n1 * 4);
    e = e ? e : A((void**)&p->pos, n1 * 4);
    e = e ? e : A((void**)&p->cellv, n1 * 4);
    e = e ? e : A((void**)&p->fa, n1 * 4);
    e = e ? e : A((void**)&p->fb, n1 * 4);
    e = e ? e : A((void**)&p->cellbuf, 3 * (((size_t)p->n_cap >> reo::CELL_SHIFT) + 2) * 4);
    e = e ? e : A((void**)&p->rcnt, 16);
    e = e ? e : A((void**)&p->dc, sizeof(DevCounters));
    if (e == cudaSuccess) e = cudaMallocHost((void**)&p->hc, sizeof(DevCounters));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ECL_SCC_ENOMEM, "plan allocation (n=%d, nnz=%lld): %s", n_max, (long long)m_max,
                    cudaGetErrorString(e));
    }
    return ECL_SCC_OK;
}

void plan_free(Plan* p) {
    for (int b = 0; b < 2; b++) {
        cudaFree(p->act[b]); cudaFree(p->cin[b]); cudaFree(p->cout[b]);
        cudaFree(p->optr[b]); cudaFree(p->iptr[b]); cudaFree(p->oadj[b]); cudaFree(p->iadj[b]);
    }
    for (int b = 0; b < 2; b++) { cudaFree(p->min_in[b]); cudaFree(p->min_out[b]); }
    cudaFree(p->t2); cudaFree(p->hpos[0]); cudaFree(p->hpos[1]); cudaFree(p->slot);
    cudaFree(p->kin); cudaFree(p->newidx); cudaFree(p->cnt); cudaFree(p->emask); cudaFree(p->sig2);
    cudaFree(p->wsum); cudaFree(p->wscan); cudaFree(p->bsum); cudaFree(p->chunks); cudaFree(p->dc);
    cudaFree(p->chunk_cnt); cudaFree(p->hcnt);
    cudaFree(p->dirty);
    cudaFree(p->rp2); cudaFree(p->ci2); cudaFree(p->orig); cudaFree(p->pos); cudaFree(p->cellv);
    cudaFree(p->fa); cudaFree(p->fb); cudaFree(p->cellbuf); cudaFree(p->rcnt);
    cudaFree(p->u_rp); cudaFree(p->u_ci); cudaFree(p->u_lab); cudaFree(p->u_desc);
    cudaFree(p->pnin); cudaFree(p->pnout); cudaFree(p->ext); cudaFree(p->ext_cnt);
    cudaFree(p->aq_state); cudaFree(p->aq_seen); cudaFree(p->aq_ctr);
    cudaFree(p->lv_ctl);
    cudaFree(p->h_rp); cudaFree(p->h_ci); cudaFree(p->h_lab);
    cudaFree(p->hb_rp); cudaFree(p->hb_ci); cudaFree(p->hb_lab);
    if (p->hc) cudaFreeHost(p->hc);
    if (p->ev_ok)
        for (int k = 0; k < 6; k++) cudaEventDestroy(p->ev[k]);
    memset(p, 0, sizeof(*p));
}

// --------------------------------------------------------------------------- scans
template <typename T>
static int scan_excl(Plan* p, const T* in, int64_t N, T* out, T* grand, void* bsum, int write_total, cudaStream_t s) {
    const int64_t nb = std::max<int64_t>(cdiv(N, SCAN_TILE), 1);
    p->launches++; k_scan_reduce<T><<<(unsigned)nb, SCAN_THREADS, 0, s>>>(in, N, (T*)bsum);
    if (nb <= SCAN_FOLD_NB) {                          // small scans: the top level folded into the apply
        p->launches++;
        k_scan_apply_fold<T><<<(unsigned)nb, SCAN_THREADS, 0, s>>>(in, N, (const T*)bsum, out, grand, write_total);
        CK(cudaGetLastError());
        return ECL_SCC_OK;
    }
    p->launches++; k_scan_top<T><<<1, SCAN_THREADS, 0, s>>>((T*)bsum, nb, grand);
    p->launches++; k_scan_apply<T><<<(unsigned)nb, SCAN_THREADS, 0, s>>>(in, N, (T*)bsum, out, grand, write_total);
    CK(cudaGetLastError());
    return ECL_SCC_OK;
}

__global__ void k_iota(int32_t n, int32_t* __restrict__ out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        out[v] = (int32_t)v;
}
// debug snapshot: signatures of the active vertices over the labels of the others
__global__ void k_scatter_sigs(int32_t na, const int32_t* __restrict__ act, const int32_t* __restrict__ cin,
                               const int32_t* __restrict__ cout, int32_t* __restrict__ din, int32_t* __restrict__ dout,
                               const int32_t* __restrict__ orig) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= na) return;
    const int v = orig ? orig[act[i]] : act[i];
    din[v] = cin[i];
    dout[v] = cout[i];
}

// --------------------------------------------------------------------------- steps
// a1: CSC of the input graph into buffer 0 (in-degree histogram, scan, scatter)
static Chunk* chunk_buf(Plan* p, int b) { return (Chunk*)p->chunks + (size_t)b * p->chunk_cap; }

static int read_nchunks(Plan* p, cudaStream_t s, int* out) {
    CK(cudaMemcpyAsync(&p->hc->nchunks, &p->dc->nchunks, sizeof(int), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (p->hc->nchunks > p->chunk_cap) return fail(ECL_SCC_ECUDA, "internal: long-row chunk list overflow");
    *out = p->hc->nchunks;
    return ECL_SCC_OK;
}
static unsigned chunk_grid(int nchunks) { return (unsigned)std::max<int64_t>(1, cdiv(nchunks, TPB / WARP)); }

// a1: CSC of the input graph into buffer 0 (in-degree histogram, scan, scatter; long
// rows by chunks) and the chunk list of the input graph (buffer p->cb)
static int build_csc(Plan* p, int32_t n, int64_t nnz, const int32_t* rp, const int32_t* ci, cudaStream_t s) {
    p->cb = 0;
    Chunk* ch = chunk_buf(p, p->cb);
    CK(cudaMemsetAsync(&p->dc->nchunks, 0, sizeof(int), s));
    CK(cudaMemsetAsync(&p->dc->maxdeg, 0, sizeof(int), s));
    p->launches++; k_ingest_chunks<<<grid_for(n, TPB), TPB, 0, s>>>(n, rp, 0, ch, &p->dc->nchunks, (int)p->chunk_cap, &p->dc->maxdeg);
    CK(cudaMemsetAsync(p->kin, 0, sizeof(int32_t) * (size_t)(n + 1), s));
    int nout = 0;
    int r = read_nchunks(p, s, &nout);
    if (r) return r;
    // graphs without long rows: per-edge ranks (in the second working buffer, free until the
    // first compaction); power-law graphs: cursor atomics (measured: returning atomics on
    // hub destinations made C3's ingest 1.8 -> 2.7 ms, while C4's went 1.22 -> 0.80 ms)
    const bool use_rank = nout == 0;
    int32_t* rank = p->oadj[1];
    int32_t* cursor = p->kout;
    const unsigned rgrid = (unsigned)std::min<int64_t>(grid_for(nnz, TPB), 148 * 8);
    p->launches++;
    if (use_rank) k_indeg_rank<true><<<rgrid, TPB, 0, s>>>(nnz, ci, p->kin, rank);
    else k_indeg_rank<false><<<rgrid, TPB, 0, s>>>(nnz, ci, p->kin, rank);
    r = scan_excl<I1>(p, (const I1*)p->kin, n, (I1*)p->iptr[0], (I1*)&p->dc->grand1, p->bsum, 1, s);
    if (r) return r;
    if (!use_rank) CK(cudaMemsetAsync(cursor, 0, sizeof(int32_t) * (size_t)n, s));
    CK(cudaMemsetAsync(&p->dc->local_e, 0, sizeof(unsigned long long), s));
    p->launches++;
    if (use_rank) k_csc_scatter<true><<<grid_for(n, TPB), TPB, 0, s>>>(n, rp, ci, p->iptr[0], rank, cursor, p->iadj[0], &p->dc->local_e);
    else k_csc_scatter<false><<<grid_for(n, TPB), TPB, 0, s>>>(n, rp, ci, p->iptr[0], rank, cursor, p->iadj[0], &p->dc->local_e);
    if (nout) { p->launches++; k_csc_scatter_chunks<false><<<chunk_grid(nout), TPB, 0, s>>>(ch, nout, ci, p->iptr[0], rank, cursor, p->iadj[0]); }
    p->launches++; k_ingest_chunks<<<grid_for(n, TPB), TPB, 0, s>>>(n, p->iptr[0], 1, ch, &p->dc->nchunks, (int)p->chunk_cap, &p->dc->maxdeg);
    CK(cudaMemcpyAsync(&p->hc->maxdeg, &p->dc->maxdeg, sizeof(int), cudaMemcpyDeviceToHost, s));
    if ((r = read_nchunks(p, s, &p->nchunks_cur))) return r;
    // the compaction's 4-byte keep words (rows <= KW_DEG entries: meshes); the variants and the
    // partitioned mode keep the general layout
    p->kw = p->hc->maxdeg <= KW_DEG && !(p->flags & (ECL_SCC_FOUR_SIG | ECL_SCC_TRIM2 | ECL_SCC_NO_KW));
    CK(cudaGetLastError());
    return ECL_SCC_OK;
}

// Storage reordering (reorder.cuh): BFS-Voronoi cells become runs of consecutive storage
// IDs; fills p->rp2 / p->ci2 (permuted CSR) and p->orig (storage -> caller ID).  Needs the
// CSC of the input (buffer 0).
static int reorder_graph(Plan* p, int32_t n, int64_t nnz, const int32_t* rp, const int32_t* ci, cudaStream_t s) {
    const unsigned gs = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
    CK(cudaMemsetAsync(p->rcnt, 0, 16, s));
    p->launches++; reo::k_seed2<<<gs, TPB, 0, s>>>(n, p->cellv, p->fa, p->rcnt);
    int h[3] = {0, 0, 0};
    for (int r = 0;; ) {
        for (int k = 0; k < 16; k++, r++) {
            p->launches++;
            reo::k_bfs_level<<<148 * 8, TPB, 0, s>>>(p->fa, p->fb, p->rcnt, r, rp, ci, p->iptr[0], p->iadj[0], p->cellv);
        }
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(h, p->rcnt, 12, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (h[r % 3] == 0) break;                      // the frontier of level r is empty
        if (r > n + 32) return fail(ECL_SCC_ECUDA, "internal: reorder BFS did not finish");
    }
    const int64_t nkeys = ((int64_t)n >> reo::CELL_SHIFT) + 1;
    int32_t* hist = p->cellbuf;
    int32_t* start = p->cellbuf + (nkeys + 1);
    int32_t* cursor = p->kout;                         // free until the first compaction
    CK(cudaMemsetAsync(hist, 0, sizeof(int32_t) * (size_t)(nkeys + 1), s));
    p->launches++; reo::k_cell_hist_agg<<<gs, TPB, 0, s>>>(n, p->cellv, hist);
    int r = scan_excl<I1>(p, (const I1*)hist, nkeys, (I1*)start, (I1*)&p->dc->grand1, p->bsum, 1, s);
    if (r) return r;
    CK(cudaMemsetAsync(cursor, 0, sizeof(int32_t) * (size_t)(nkeys + 1), s));
    p->launches++; reo::k_cell_place<<<gs, TPB, 0, s>>>(n, p->cellv, start, cursor, p->pos, p->orig);
    int bits = 1;
    while (bits < 31 && (1ll << bits) <= (long long)n) bits++;   // every caller ID < 2^bits - 1
    p->launches++;
    reo::k_cell_sort<<<(unsigned)std::min<int64_t>(nkeys, 148 * 8), reo::SORT_THREADS, 0, s>>>(nkeys, start, p->orig, p->pos, bits);
    p->launches++; reo::k_perm_deg<<<gs, TPB, 0, s>>>(n, rp, p->pos, p->kin);
    r = scan_excl<I1>(p, (const I1*)p->kin, n, (I1*)p->rp2, (I1*)&p->dc->grand1, p->bsum, 1, s);
    if (r) return r;
    p->launches++; reo::k_perm_fill<<<grid_for(n, TPB), TPB, 0, s>>>(n, rp, ci, p->pos, p->rp2, p->ci2);
    CK(cudaGetLastError());
    (void)nnz;
    return ECL_SCC_OK;
}

// Does Phase 2 of a working graph with `nchunks` long-row chunks run on tile packs?
static bool pack_path(const Plan* p, int nchunks) {
    const bool sync = (p->flags & ECL_SCC_SYNC_PASSES) != 0 || (p->low_locality && nchunks > 0);
    return nchunks == 0 && !sync && !(p->flags & (ECL_SCC_NO_DIRTY | ECL_SCC_NO_PACK | ECL_SCC_CLUSTER));
}
// Does Phase 2 run on cluster pair tiles (cluster.cuh)?
static bool cluster_path(const Plan* p, int nchunks) {
    return (p->flags & ECL_SCC_CLUSTER) && nchunks == 0 &&
           !(p->flags & (ECL_SCC_SYNC_PASSES | ECL_SCC_NO_DIRTY | ECL_SCC_NO_PACK | ECL_SCC_NO_ASYNC));
}
// tile pack buffers (pack.cuh), sized for the plan on first use
static int ensure_pack(Plan* p) {
    if (p->pnin) return ECL_SCC_OK;
    const size_t np = (size_t)cdiv((int64_t)p->n_cap + 1, PACK_TT) * PACK_TT + PACK_TT;
    cudaError_t e = cudaMalloc((void**)&p->pnin, np * 8);
    if (e == cudaSuccess) e = cudaMalloc((void**)&p->pnout, np * 8);
    if (e == cudaSuccess) e = cudaMalloc((void**)&p->ext, 2 * (size_t)p->m_cap * sizeof(int2) + 16);
    if (e == cudaSuccess) e = cudaMalloc((void**)&p->ext_cnt, (size_t)p->dirty_cap * 4);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ECL_SCC_ENOMEM, "tile pack allocation: %s", cudaGetErrorString(e));
    }
    for (auto kf : {k_prop_pack<false>, k_prop_pack<true>}) {
        CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pack_dyn_smem()));
        CK(cudaFuncSetAttribute(kf, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared));
    }
    return ECL_SCC_OK;
}

// a7 + a2 + a3 + a8: Phase 3 edge removal, Trim-1, compaction into buffer `ob` with the
// Phase-1 reset of the survivors and the final labels of the vertices that leave.  Two
// parts: compact_keep evaluates the keep predicate (kept degrees), compact_finish trims and
// compacts; the partitioned mode exchanges the halo's kept degrees in between.
template <bool FIRST, bool TRIM, bool FOUR, bool KW = false>
static int compact_keep(Plan* p, const WGraph& g, const int32_t* cin, const int32_t* cout, cudaStream_t s) {
    const unsigned grid = grid_for(g.na, TPB);
    const int nc = p->nchunks_cur, chunked = nc > 0;
    const Chunk* cur = chunk_buf(p, p->cb);
    CK(cudaMemsetAsync(&p->dc->nchunks, 0, sizeof(int), s));
    CK(cudaMemsetAsync(&p->dc->pack_bad, 0, sizeof(int), s));
    // power-law graphs (long-row chunks): keep() gathers random far ends, so the two signature
    // arrays are interleaved once (one gather per far end instead of two)
    WGraph gk = g;
    if (!FIRST && chunked) {
        p->launches++;
        k_pack_sig<<<std::min<unsigned>(grid, 148 * 16), TPB, 0, s>>>(g.na, cin, cout, p->sig2);
        gk.sig2 = p->sig2;
    }
    p->launches++; k_keep_count<FIRST, FOUR, KW><<<grid, TPB, 0, s>>>(gk, cin, cout, p->kio, chunked, p->hcnt, p->emask);
    if (chunked) {
        p->launches++;
        k_keep_chunks<FIRST, FOUR><<<chunk_grid(nc), TPB, 0, s>>>(gk, cur, nc, cin, cout, p->kio);
    }
    p->gk = gk;
    CK(cudaGetLastError());
    return ECL_SCC_OK;
}

template <bool FIRST, bool TRIM, bool FOUR, bool KW = false>
static int compact_finish(Plan* p, const int32_t* cin, const int32_t* cout, int ob, int32_t* labels, const Prio& P,
                          cudaStream_t s) {
    const WGraph gk = p->gk;
    const unsigned grid = grid_for(gk.na, TPB);
    const int64_t nw = (int64_t)grid * (TPB / WARP);
    const int nc = p->nchunks_cur, chunked = nc > 0;
    const Chunk* cur = chunk_buf(p, p->cb);
    // the scatter writes the next graph's tile pack when Phase 2 will use one (no long rows
    // now means none after the compaction)
    PackOut pk{nullptr, nullptr, nullptr, nullptr, &p->dc->pack_bad};
    p->pack_fused = pack_path(p, nc);
    if (p->pack_fused) {
        if (int r = ensure_pack(p)) return r;
        pk = PackOut{p->pnin, p->pnout, p->ext, p->ext_cnt, &p->dc->pack_bad};
    }
    const bool trim2 = TRIM && (p->flags & ECL_SCC_TRIM2);
    if (trim2) {                                   // Trim-2 on the kept degrees (reading 17)
        p->launches += 2;
        k_trim2_find<FIRST, FOUR><<<grid, TPB, 0, s>>>(gk, cin, cout, p->kio, p->emask, p->t2);
        k_trim2_apply<<<grid, TPB, 0, s>>>(gk.na, p->t2, p->kio);
    }
    if (chunked) {
        p->launches++;
        k_count_chunks<FIRST, TRIM, FOUR><<<chunk_grid(nc), TPB, 0, s>>>(gk, cur, nc, cin, cout, p->kio, p->chunk_cnt, p->hcnt);
    }
    p->launches++;
    if (KW && !FOUR)                                   // keep words: two lane-strided vertices per thread
        k_compact_count2<FIRST, TRIM><<<(unsigned)cdiv(nw * WARP / CNT2, TPB), TPB, 0, s>>>(gk, cin, cout, (uint32_t*)p->emask,
                                                                                           p->wsum, nw);
    else
        k_compact_count<FIRST, TRIM, FOUR, KW><<<grid, TPB, 0, s>>>(gk, cin, cout, p->kio, p->cnt, p->wsum, chunked, p->hcnt, p->emask);
    int r = scan_excl<I3>(p, (const I3*)p->wsum, nw, (I3*)p->wscan, (I3*)&p->dc->totals, p->bsum, 0, s);
    if (r) return r;
    if (KW && !trim2 && !p->min_in[ob]) {               // keep words: four vertices per thread
        p->launches++;
        k_compact_map4<FIRST><<<(unsigned)cdiv(cdiv((int64_t)gk.na, MAP4 * WARP) * WARP, TPB), TPB, 0, s>>>(
            gk, cin, cout, (const uint32_t*)p->emask, p->wscan, &p->dc->totals, p->newidx, p->act[ob], p->cin[ob],
            p->cout[ob], p->optr[ob], p->iptr[ob], labels, P, p->orig_cur, pk,
            MapExtra{nullptr, nullptr, nullptr, p->kio, TRIM ? 1 : 0, gk.hpos ? p->hpos[ob] : nullptr, p->lab_lo,
                     p->lab_hi, p->slot});
    } else {
    p->launches++; k_compact_map<FIRST, KW><<<grid, TPB, 0, s>>>(gk, cin, cout, KW ? (const int2*)p->emask : p->cnt, p->wscan, &p->dc->totals, p->newidx, p->act[ob],
                                              p->cin[ob], p->cout[ob], p->optr[ob], p->iptr[ob], labels,
                                              chunk_buf(p, p->cb ^ 1), &p->dc->nchunks, (int)p->chunk_cap, P, p->orig_cur, pk,
                                              MapExtra{p->min_in[ob], p->min_out[ob], trim2 ? p->t2 : nullptr, p->kio,
                                                       TRIM ? 1 : 0, gk.hpos ? p->hpos[ob] : nullptr, p->lab_lo,
                                                       p->lab_hi, p->slot});
    }
    p->launches++; k_compact_scatter<FIRST, TRIM, FOUR, KW><<<grid, TPB, 0, s>>>(gk, cin, cout, p->kio, p->newidx, p->optr[ob],
                                                          p->iptr[ob], p->oadj[ob], p->iadj[ob], chunked, p->emask, pk);
    if (chunked) {
        p->launches++;
        k_scatter_chunks<FIRST, TRIM, FOUR><<<chunk_grid(nc), TPB, 0, s>>>(gk, cur, nc, cin, cout, p->kio, p->chunk_cnt,
                                                                     p->newidx, p->optr[ob], p->iptr[ob], p->oadj[ob], p->iadj[ob]);
    }
    p->cb ^= 1;                                   // the next graph's chunk list is now current
    CK(cudaGetLastError());
    return ECL_SCC_OK;
}

// part 0 = keep, 1 = finish, of the compaction before outer iteration `iter`
static int compaction(Plan* p, int part, int iter, const WGraph& g, const int32_t* cin, const int32_t* cout, int ob,
                      int32_t* labels, const Prio& P, cudaStream_t s) {
    const bool trim = !(p->flags & ECL_SCC_NO_TRIM);
    const bool four = (p->flags & ECL_SCC_FOUR_SIG) != 0 && iter > 1;   // (iteration 1 keeps every edge)
#define ECL_COMPACT(F, T, Fo) \
    return part == 0 ? compact_keep<F, T, Fo>(p, g, cin, cout, s) : compact_finish<F, T, Fo>(p, cin, cout, ob, labels, P, s)
#define ECL_COMPACT_KW(F, T) \
    return part == 0 ? compact_keep<F, T, false, true>(p, g, cin, cout, s) \
                     : compact_finish<F, T, false, true>(p, cin, cout, ob, labels, P, s)
    if (p->kw && !g.hpos) {                        // small degrees (the partitioned mode excluded)
        if (iter == 1) {
            if (trim) ECL_COMPACT_KW(true, true);
            ECL_COMPACT_KW(true, false);
        }
        if (trim) ECL_COMPACT_KW(false, true);
        ECL_COMPACT_KW(false, false);
    }
    if (iter == 1) {
        if (trim) ECL_COMPACT(true, true, false);
        ECL_COMPACT(true, false, false);
    }
    if (four) {
        if (trim) ECL_COMPACT(false, true, true);
        ECL_COMPACT(false, false, true);
    }
    if (trim) ECL_COMPACT(false, true, false);
    ECL_COMPACT(false, false, false);
#undef ECL_COMPACT
#undef ECL_COMPACT_KW
}

// per-plan (per-device) kernel attributes of the pass kernels
static int set_tile_attrs(Plan* p) {
    if (p->tile_attrs) return ECL_SCC_OK;
    CK(cudaFuncSetAttribute(k_prop_tile<false, TILE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tile_dyn_smem<TILE>()));
    CK(cudaFuncSetAttribute(k_prop_tile<true, TILE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tile_dyn_smem<TILE>()));
    p->tile_attrs = true;
    return ECL_SCC_OK;
}

// runs of consecutive tiles per CTA (Gauss-Seidel along a run).  Measured on C4: run 4
// beats 1 (-14%), longer runs starve the SMs (fewer CTAs than resident slots).
static int pass_run(const Plan* p, int64_t ntiles) {
    return (int)std::min<int64_t>(p->knob_run ? p->knob_run : 4, std::max<int64_t>(1, ntiles / (2 * 148)));
}

static int launch_tile(Plan* p, bool sync, const WGraph& g, int32_t* cin, int32_t* cout, int pass, int first,
                       uint8_t* dcur, uint8_t* dnext, int full, cudaStream_t s) {
    if (int r = set_tile_attrs(p)) return r;
    const int64_t ntiles = cdiv(g.na, TILE);
    const int run = pass_run(p, ntiles);
    const unsigned grid = (unsigned)cdiv(ntiles, run);
    p->launches++;
    if (sync) k_prop_tile<true, TILE><<<grid, TILE / VPT, tile_dyn_smem<TILE>(), s>>>(g, cin, cout, p->dc, pass, first, nullptr, nullptr, 1, run);
    else k_prop_tile<false, TILE><<<grid, TILE / VPT, tile_dyn_smem<TILE>(), s>>>(g, cin, cout, p->dc, pass, first, dcur, dnext, full, run);
    return ECL_SCC_OK;
}

// the asynchronous Phase-2 queue (pack.cuh AsyncQ) and k_prop_async's launch attributes, on first use
static int ensure_async(Plan* p) {
    if (p->aq_state) return ECL_SCC_OK;
    const size_t nt = (size_t)p->dirty_cap;
    cudaError_t e = cudaMalloc((void**)&p->aq_state, nt * 4);
    if (e == cudaSuccess) e = cudaMalloc((void**)&p->aq_seen, nt);
    if (e == cudaSuccess) e = cudaMalloc((void**)&p->aq_ctr, AQ_WORDS * sizeof(unsigned long long));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ECL_SCC_ENOMEM, "async queue allocation: %s", cudaGetErrorString(e));
    }
    for (auto kf : {k_prop_async<false, false>, k_prop_async<true, false>, k_prop_async<false, true>}) {
        CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pack_dyn_smem()));
        CK(cudaFuncSetAttribute(kf, cudaFuncAttributePreferredSharedMemoryCarveout,
                                (int)cudaSharedmemCarveoutMaxShared));
    }
    int per_sm = 0, sms = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_prop_async<false, false>, PACK_TH, pack_dyn_smem()));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device));
    // resident CTAs per SM used (<= what fits); measured best: all of them
    if (p->knob_async_ctas) per_sm = std::min(per_sm, p->knob_async_ctas);
    p->aq_resident = (int64_t)std::max(1, per_sm) * sms;
    if (getenv("ECL_SCC_DEBUG")) fprintf(stderr, "[ecl_scc] k_prop_async: %d CTAs per SM\n", per_sm);
    return ECL_SCC_OK;
}

// a4-a6: Phase 2 to its fixed point.  Passes are enqueued in growing batches; a pass
// whose predecessor changed nothing exits at once, so over-enqueueing costs only a launch.
// second: a second fixed point over the same graph (the minimum pair); push: the
// partitioned mode's halo pushes; resume: continue after the halo exchange re-opened tiles
// (their state / dirty flags set by k_halo_apply) instead of starting with every tile
static int propagate(Plan* p, const WGraph& g, int32_t* cin, int32_t* cout, int nchunks, cudaStream_t s,
                     int64_t* passes_out, bool second = false, const HaloPush* push = nullptr, bool resume = false) {
    const unsigned ntiles = (unsigned)cdiv(g.na, TILE);
    const unsigned hgrid = (unsigned)std::min<int64_t>(cdiv(std::max(nchunks, 1), TPB / WARP), 148 * 8);
    // plain Jacobi passes: the ablation flag, or graphs whose tiles hold almost no edges
    const bool sync = (p->flags & ECL_SCC_SYNC_PASSES) != 0 || (p->low_locality && nchunks > 0);
    // dirty-tile skipping needs every raise to be seen by the tile kernel (no heavy rows)
    // and a local fixed point per visit (not the SYNC ablation)
    const bool use_dirty = nchunks == 0 && !sync && !(p->flags & ECL_SCC_NO_DIRTY);
    uint8_t* D[2] = {p->dirty, p->dirty + p->dirty_cap};
    if (cluster_path(p, nchunks) && g.na > 0) {          // thread-block-cluster pair tiles (cluster.cuh)
        if (int r = ensure_pack(p)) return r;
        const unsigned npair = (unsigned)cdiv(g.na, PAIR_TT);
        if (!p->aq_state) {
            const size_t nt = (size_t)p->dirty_cap;
            cudaError_t e = cudaMalloc((void**)&p->aq_state, nt * 4);
            if (e == cudaSuccess) e = cudaMalloc((void**)&p->aq_seen, nt);
            if (e == cudaSuccess) e = cudaMalloc((void**)&p->aq_ctr, AQ_WORDS * sizeof(unsigned long long));
            if (e != cudaSuccess) {
                cudaGetLastError();
                return fail(ECL_SCC_ENOMEM, "async queue allocation: %s", cudaGetErrorString(e));
            }
            CK(cudaFuncSetAttribute(k_prop_cluster, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pack_dyn_smem()));
            CK(cudaFuncSetAttribute(k_prop_cluster, cudaFuncAttributePreferredSharedMemoryCarveout,
                                    (int)cudaSharedmemCarveoutMaxShared));
            int per_sm = 0, sms = 0;
            CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_prop_cluster, PACK_TH, pack_dyn_smem()));
            CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device));
            p->aq_resident = std::max<int64_t>(2, ((int64_t)std::max(1, per_sm) * sms) & ~1ll);
        }
        if (!second) {
            p->launches++;
            k_pack_pair<<<npair, PACK_TH, 0, s>>>(g, p->pnin, p->pnout, p->ext, p->ext_cnt);
            CK(cudaMemsetAsync(&p->dc->err, 0, sizeof(int), s));
            CK(cudaMemsetAsync(&p->dc->passes, 0, sizeof(unsigned long long), s));
        }
        AsyncQ Q{p->aq_state, p->aq_seen, p->aq_ctr};
        const int64_t clusters = p->aq_resident / 2;
        const int claim = p->knob_claim ? p->knob_claim : (int)std::min<int64_t>(16, std::max<int64_t>(1, npair / clusters));
        p->launches += 2;
        k_async_init<<<grid_for((int64_t)npair, TPB), TPB, 0, s>>>(Q, (int)npair);
        const unsigned cgrid = (unsigned)(2 * std::min<int64_t>(npair, clusters));
        k_prop_cluster<<<cgrid, PACK_TH, pack_dyn_smem(), s>>>(g, cin, cout, p->pnin, p->pnout, p->ext, p->ext_cnt,
                                                               p->dc, Q, claim);
        CK(cudaGetLastError());
        *passes_out = -(int64_t)npair;
        return ECL_SCC_OK;
    }
    // tile packs (pack.cuh): the default for graphs without long rows
    const bool use_pack = pack_path(p, nchunks) && g.na > 0;
    if (use_pack) {
        if (int r = ensure_pack(p)) return r;
        if (!second && !resume && (!p->pack_fused || p->hc->pack_bad)) {   // the scatter did not write it
            p->launches++;
            k_tile_pack<<<ntiles, PACK_TH, 0, s>>>(g, p->pnin, p->pnout, p->ext, p->ext_cnt);
        }
        CK(cudaGetLastError());
        if (!(p->flags & ECL_SCC_NO_ASYNC)) {          // one persistent launch (pack.cuh)
            if (int r = ensure_async(p)) return r;
            AsyncQ Q{p->aq_state, p->aq_seen, p->aq_ctr};
            // tiles per claim: runs pay when there are many tiles per resident CTA (measured:
            // C4 iteration 1, 18 tiles per CTA, best at 8-16; C2, ~1 tile per CTA, best at 1);
            // claim = clamp(tiles / resident CTAs, 1, 16) (C4 lex 19.8 -> 19.2 ms vs
            // tiles / (2 x resident) capped at 8; blocked8 unchanged)
            const int cdiv_ = p->knob_claim_div ? p->knob_claim_div : 1;
            const int cmax = p->knob_claim_max ? p->knob_claim_max : 16;
            const int claim = p->knob_claim ? p->knob_claim
                                            : (int)std::min<int64_t>(cmax, std::max<int64_t>(1, ntiles / (cdiv_ * p->aq_resident)));
            if (!second && !resume) {
                CK(cudaMemsetAsync(&p->dc->err, 0, sizeof(int), s));
                CK(cudaMemsetAsync(&p->dc->passes, 0, sizeof(unsigned long long), s));
            }
            if (resume) {                                // cursor and stop words; pending came with the marks
                CK(cudaMemsetAsync(p->aq_ctr + AQ_CUR, 0, sizeof(unsigned long long), s));
                CK(cudaMemsetAsync(p->aq_ctr + AQ_STOP, 0, sizeof(unsigned long long), s));
            } else {
                p->launches++;
                k_async_init<<<grid_for((int64_t)ntiles, TPB), TPB, 0, s>>>(Q, (int)ntiles);
            }
            p->launches++;
            const unsigned agrid = (unsigned)std::min<int64_t>(ntiles, p->aq_resident);
            if (push) k_prop_async<true, false><<<agrid, PACK_TH, pack_dyn_smem(), s>>>(
                g, cin, cout, p->pnin, p->pnout, p->ext, p->ext_cnt, p->dc, Q, claim, *push);
            else if (g.compress | g.raise_) k_prop_async<false, true><<<agrid, PACK_TH, pack_dyn_smem(), s>>>(
                g, cin, cout, p->pnin, p->pnout, p->ext, p->ext_cnt, p->dc, Q, claim, HaloPush{});
            else k_prop_async<false, false><<<agrid, PACK_TH, pack_dyn_smem(), s>>>(
                g, cin, cout, p->pnin, p->pnout, p->ext, p->ext_cnt, p->dc, Q, claim, HaloPush{});
            CK(cudaGetLastError());
            // no stream synchronisation here: the watchdog word and the visit count are read
            // with the counters of the next compaction (resolve_prop in run_graph)
            *passes_out = -(int64_t)ntiles;
            return ECL_SCC_OK;
        }
    }
    CK(cudaMemsetAsync(p->dc->changed, 0, sizeof(int) * RING, s));
    CK(cudaMemsetAsync(&p->dc->passes, 0, sizeof(unsigned long long), s));
    if (use_dirty) {
        if (!resume) CK(cudaMemsetAsync(D[0], 1, ntiles, s));   // (resume: k_halo_apply's flags)
        CK(cudaMemsetAsync(D[1], 0, ntiles, s));
    }
    int pass = 0;
    int batch = 2;
    for (;;) {
        for (int k = 0; k < batch; k++, pass++) {
            uint8_t* dc_ = use_dirty ? D[pass & 1] : nullptr;
            uint8_t* dn_ = use_dirty ? D[(pass + 1) & 1] : nullptr;
            if (nchunks) { p->launches++; k_prop_heavy<<<hgrid, TPB, 0, s>>>(chunk_buf(p, p->cb), nchunks, g, cin, cout, p->dc, pass); }
            const int full = (pass == 0 || nchunks > 0);
            if (use_pack) {
                const int run = pass_run(p, ntiles);
                p->launches++;
                if (g.compress | g.raise_)
                    k_prop_pack<true><<<(unsigned)cdiv(ntiles, run), PACK_TH, pack_dyn_smem(), s>>>(
                        g, cin, cout, p->pnin, p->pnout, p->ext, p->ext_cnt, p->dc, pass, nchunks == 0, dc_, dn_, full, run);
                else
                    k_prop_pack<false><<<(unsigned)cdiv(ntiles, run), PACK_TH, pack_dyn_smem(), s>>>(
                        g, cin, cout, p->pnin, p->pnout, p->ext, p->ext_cnt, p->dc, pass, nchunks == 0, dc_, dn_, full, run);
                continue;
            }
            if (int r = launch_tile(p, sync, g, cin, cout, pass, nchunks == 0, dc_, dn_, full, s)) return r;
        }
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (p->hc->changed[(pass - 1) & (RING - 1)] == 0) break;
        // a monotone max over int32 IDs cannot take more passes than this
        if ((int64_t)pass > 4 * (int64_t)g.na + 1024)
            return fail(ECL_SCC_ECUDA, "internal: Phase 2 did not converge after %d passes", pass);
        batch = std::min(batch * 2, RING / 2);
    }
    if (getenv("ECL_SCC_DEBUG"))
        fprintf(stderr, "[ecl_scc] na=%d passes=%llu visited_vertices=%llu\n", g.na,
                (unsigned long long)p->hc->passes, (unsigned long long)p->hc->visit_v);
    *passes_out = (int64_t)p->hc->passes;
    if (push && g.na > 0) {                       // pass kernels: push every halo copy afterwards
        p->launches++;
        k_halo_push<<<std::min<unsigned>(grid_for(g.na, TPB), 148 * 8), TPB, 0, s>>>(g.na, cin, cout, *push);
        CK(cudaGetLastError());
    }
    return ECL_SCC_OK;
}

// the deferred check of an asynchronous Phase 2 (propagate() returned -ntiles as its pass
// count): after a stream synchronisation p->hc holds its watchdog word and visit count
static int resolve_prop(Plan* p, int64_t* passes) {
    if (*passes >= 0) return ECL_SCC_OK;
    const int64_t ntiles = -*passes;
    if (p->hc->err == 3) return fail(ECL_SCC_ECUDA, "internal: asynchronous Phase 2 stalled (watchdog)");
    *passes = cdiv((int64_t)p->hc->passes, ntiles);              // sweep equivalents
    return ECL_SCC_OK;
}

// stage timing: events 2k/2k+1 bracket stage k (0 ingest, 1 compaction, 2 Phase 2)
static void stage_mark(Plan* p, int ev, cudaStream_t s) {
    if (!(p->flags & ECL_SCC_TIME_STAGES)) return;
    if (!p->ev_ok) {
        for (int k = 0; k < 6; k++) cudaEventCreate(&p->ev[k]);
        p->ev_ok = true;
    }
    cudaEventRecord(p->ev[ev], s);
}
static double stage_ms(Plan* p, int k) {   // call after a stream sync
    if (!(p->flags & ECL_SCC_TIME_STAGES) || !p->ev_ok) return 0.0;
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, p->ev[2 * k], p->ev[2 * k + 1]) != cudaSuccess) { cudaGetLastError(); return 0.0; }
    return (double)ms;
}

// the whole path for one (possibly union) graph; labels_out receives the result
int run_graph(Plan* p, int32_t n, int64_t nnz, const int32_t* rp, const int32_t* ci, int32_t* labels,
              cudaStream_t s, ecl_scc_stats* st, int stop_iter, int32_t* dbg_in, int32_t* dbg_out) {
    if (st) memset(st, 0, sizeof(*st));
    CK(cudaMemsetAsync(p->dc->prof, 0, sizeof(p->dc->prof) + 3 * sizeof(unsigned long long), s));
    stage_mark(p, 0, s);
    if (!(p->flags & ECL_SCC_NO_VALIDATE) && n > 0) {
        CK(cudaMemsetAsync(&p->dc->err, 0, sizeof(int), s));
        p->launches++; k_validate<<<std::min<unsigned>(grid_for(std::max<int64_t>(n, nnz), TPB), 148 * 16), TPB, 0, s>>>(n, nnz, rp, ci, &p->dc->err);
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (p->hc->err) return fail(ECL_SCC_ERANGE, "invalid CSR: offsets not monotone from 0 to nnz, or column outside [0,n)");
    }
    const Prio P = make_prio((uint32_t)n, (p->flags & ECL_SCC_IDENTITY_IDS) != 0);
    int iters = 0;
    bool stopped = false;
    if (nnz == 0) {
        p->launches++; k_iota<<<grid_for(n, TPB), TPB, 0, s>>>(n, labels);      // Alg. 1 l.3-6, nothing to remove
        CK(cudaGetLastError());
    } else {
        // the debug snapshot reads every label slot; start from a defined value
        if (stop_iter > 0) CK(cudaMemsetAsync(labels, 0, sizeof(int32_t) * (size_t)n, s));
        int r = build_csc(p, n, nnz, rp, ci, s);
        if (r) return r;
        p->orig_cur = nullptr;
        // storage reordering for graphs without long rows (meshes) whose numbering keeps
        // fewer than REORDER_LOCALITY of the edges inside 2048-ID ranges; results do not
        // depend on it, only the number of Phase-2 passes does
        bool reorder = false;
        unsigned long long loc = 0;                     // edges inside 2048-ID ranges
        CK(cudaMemcpyAsync(&loc, &p->dc->local_e, sizeof(loc), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        p->low_locality = (double)loc < LOCAL_FP_LOCALITY * (double)nnz;
        if ((p->flags & ECL_SCC_FORCE_REORDER) && p->nchunks_cur == 0) reorder = true;
        else if (!(p->flags & ECL_SCC_NO_REORDER) && p->nchunks_cur == 0 && n >= REORDER_MIN_N)
            reorder = (double)loc < REORDER_LOCALITY * (double)nnz;
        if (reorder) p->low_locality = false;
        if (reorder) {
            if ((r = reorder_graph(p, n, nnz, rp, ci, s))) return r;
            rp = p->rp2;
            ci = p->ci2;
            if ((r = build_csc(p, n, nnz, rp, ci, s))) return r;
            p->orig_cur = p->orig;
        }
        stage_mark(p, 1, s);
        WGraph g{nullptr, rp, ci, p->iptr[0], p->iadj[0], n};
        const int32_t *cin = nullptr, *cout = nullptr;          // identity (l.3-6) in the input
        int ob = 1;
        int64_t pend_passes = 0;                                 // deferred Phase-2 check
        int pend_iter = 0;
        auto resolve = [&]() -> int {
            if (!pend_iter) return ECL_SCC_OK;
            if (int e = resolve_prop(p, &pend_passes)) return e;
            if (st) {
                if (pend_iter - 1 < ECL_SCC_TRACE_MAX) st->passes_iter[pend_iter - 1] = pend_passes;
                st->passes += pend_passes;
            }
            pend_iter = 0;
            return ECL_SCC_OK;
        };
        for (int iter = 1;; iter++) {
            if (iter > n + 2) return fail(ECL_SCC_ECUDA, "internal: outer loop exceeded n+2 iterations");
            stage_mark(p, 2, s);
            r = compaction(p, 0, iter, g, cin, cout, ob, labels, P, s);
            if (!r) r = compaction(p, 1, iter, g, cin, cout, ob, labels, P, s);
            if (r) return r;
            stage_mark(p, 3, s);
            CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
            CK(cudaStreamSynchronize(s));
            if ((r = resolve())) return r;
            if (st) {
                if (iter == 1) st->ms_ingest += stage_ms(p, 0);
                const double mc = stage_ms(p, 1);
                st->ms_compact += mc;
                if (iter - 1 < ECL_SCC_TRACE_MAX) st->ms_compact_iter[iter - 1] = mc;
            }
            const int4 t = p->hc->totals;
            const int nchunks = p->hc->nchunks;
            p->nchunks_cur = nchunks;
            // kept edges (before trim) = the kept out-degrees summed by the compaction scan
            if (st && iter >= 2 && iter - 2 < ECL_SCC_TRACE_MAX) st->edges_kept[iter - 2] = (int64_t)p->hc->totals.w;
            if (t.y != t.z) return fail(ECL_SCC_ECUDA, "internal: CSR/CSC survivor mismatch %d vs %d", t.y, t.z);
            if (nchunks > p->chunk_cap) return fail(ECL_SCC_ECUDA, "internal: heavy chunk list overflow");
            g = WGraph{p->act[ob], p->optr[ob], p->oadj[ob], p->iptr[ob], p->iadj[ob], t.x, nullptr,
                       p->min_in[ob], p->min_out[ob]};
            g.slot = p->slot;
            g.compress = (p->flags & ECL_SCC_COMPRESS) ? 1 : 0;
            g.raise_ = (p->flags & ECL_SCC_RAISE) ? 1 : 0;
            cin = p->cin[ob];
            cout = p->cout[ob];
            if (t.y == 0) break;                                   // no live edge: done
            int64_t passes = 0;
            stage_mark(p, 4, s);
            r = propagate(p, g, p->cin[ob], p->cout[ob], nchunks, s, &passes);
            if (r) return r;
            if (p->flags & ECL_SCC_FOUR_SIG) {            // the minimum pair: its own fixed point
                int64_t p2 = 0;
                r = propagate(p, g, p->min_in[ob], p->min_out[ob], nchunks, s, &p2, true);
                if (r) return r;
                if (passes >= 0) passes += p2;           // (asynchronous: counted on the device)
            }
            stage_mark(p, 5, s);
            if (st && (p->flags & ECL_SCC_TIME_STAGES)) {
                CK(cudaEventSynchronize(p->ev[5]));
                const double mp = stage_ms(p, 2);
                st->ms_prop += mp;
                if (iter - 1 < ECL_SCC_TRACE_MAX) st->ms_prop_iter[iter - 1] = mp;
            }
            iters = iter;
            if (st && iter - 1 < ECL_SCC_TRACE_MAX) {
                st->edges_in[iter - 1] = t.y;
                st->vertices_in[iter - 1] = t.x;
            }
            pend_passes = passes;
            pend_iter = iter;
            if (passes >= 0 || (p->flags & ECL_SCC_TIME_STAGES)) {   // already synchronised
                if ((p->flags & ECL_SCC_TIME_STAGES) && passes < 0) {
                    CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
                    CK(cudaStreamSynchronize(s));
                }
                if ((r = resolve())) return r;
            }
            if (stop_iter == iter) {
                CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
                CK(cudaStreamSynchronize(s));
                if ((r = resolve())) return r;
                p->launches++; k_snapshot_left<<<grid_for(n, TPB), TPB, 0, s>>>(n, labels, dbg_in, dbg_out, P);
                p->launches++; k_scatter_sigs<<<grid_for(t.x, TPB), TPB, 0, s>>>(t.x, g.act, cin, cout, dbg_in, dbg_out, p->orig_cur);
                CK(cudaGetLastError());
                stopped = true;
                break;
            }
            ob ^= 1;
        }
        if (!P.ids && !stopped) {
            // labels of finished vertices are still max priorities: map to max vertex IDs
            const unsigned gr = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
            CK(cudaMemsetAsync(p->kin, 0xFF, sizeof(int32_t) * (size_t)n, s));
            p->launches++; k_relabel_fold<<<gr, TPB, 0, s>>>(n, labels, p->kin);
            p->launches++; k_relabel_apply<<<gr, TPB, 0, s>>>(n, labels, p->kin);
            CK(cudaGetLastError());
        }
    }
    if (stop_iter > 0 && !stopped) {
        CK(cudaMemcpyAsync(dbg_in, labels, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpyAsync(dbg_out, labels, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToDevice, s));
    }
    CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (st) {
        st->iterations = iters;
        st->trace_len = std::min(iters, ECL_SCC_TRACE_MAX);
        st->kernel_launches = p->launches;
        // SURVEY 8(d) accounting over the tiles actually visited: 4 B offset + 16 B own
        // in/out read+write per vertex, 12 B per edge (index + both far-end signatures);
        // heavy chunks: 8 B per edge (index + one far-end signature)
        st->prop_bytes = (int64_t)(20 * p->hc->visit_v + 12 * p->hc->visit_e + 8 * p->hc->heavy_e);
    }
    return ECL_SCC_OK;
}

// --------------------------------------------------------------------------- batched union
__global__ void k_set1(int32_t* p, int32_t v) { *p = v; }
// all graphs of a batch in one launch (blockIdx.y = graph): the union rows and columns, with
// the CSR checks of k_validate on the way (one pass over every input); and the label split
struct UGraph {
    const int32_t* rp;
    const int32_t* ci;
    int32_t* lab;
    int64_t nnz, eoff;
    int32_t n, voff;
};
__global__ void k_union_all(const UGraph* __restrict__ gs, int32_t* __restrict__ urp, int32_t* __restrict__ uci,
                            int validate, int* __restrict__ err) {
    const UGraph G = gs[blockIdx.y];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int bad = 0;
    for (int64_t v = t0; v < G.n; v += stride) {
        const int32_t a = G.rp[v];
        urp[G.voff + v] = a + (int32_t)G.eoff;
        if (validate) {
            const int32_t b = G.rp[v + 1];
            if (a > b || (v == 0 && a != 0) || (v == G.n - 1 && (int64_t)b != G.nnz)) bad = 1;
        }
    }
    for (int64_t e = t0; e < G.nnz; e += stride) {
        const int32_t c = G.ci[e];
        if (validate && (c < 0 || c >= G.n)) bad = 1;
        uci[G.eoff + e] = c + G.voff;
    }
    if (bad) *err = 1;
}
__global__ void k_split_all(const UGraph* __restrict__ gs, const int32_t* __restrict__ ul) {
    const UGraph G = gs[blockIdx.y];
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < G.n; v += (int64_t)gridDim.x * blockDim.x)
        G.lab[v] = ul[G.voff + v] - G.voff;
}

int run_batched(Plan* p, int32_t G, const int32_t* n, const int64_t* nnz, const int32_t* const* rp,
                const int32_t* const* ci, int32_t* const* labels, cudaStream_t s, ecl_scc_stats* st) {
    int64_t N = 0, M = 0;
    for (int g = 0; g < G; g++) { N += n[g]; M += nnz[g]; }
    p->launches = 0;
    if (!p->u_rp || p->u_n_cap < N) {
        cudaFree(p->u_rp);
        cudaFree(p->u_lab);
        p->u_rp = p->u_lab = nullptr;
        if (cudaMalloc((void**)&p->u_rp, sizeof(int32_t) * (size_t)(N + 1)) != cudaSuccess ||
            cudaMalloc((void**)&p->u_lab, sizeof(int32_t) * (size_t)(N + 1)) != cudaSuccess) {
            cudaGetLastError();
            return fail(ECL_SCC_ENOMEM, "batched union offsets (%lld vertices)", (long long)N);
        }
        p->u_n_cap = N;
    }
    if (!p->u_ci || p->u_m_cap < M) {
        cudaFree(p->u_ci);
        p->u_ci = nullptr;
        if (cudaMalloc((void**)&p->u_ci, sizeof(int32_t) * (size_t)std::max<int64_t>(M, 1)) != cudaSuccess) {
            cudaGetLastError();
            return fail(ECL_SCC_ENOMEM, "batched union columns (%lld edges)", (long long)M);
        }
        p->u_m_cap = M;
    }
    // one launch builds the union (and checks every graph's CSR on the way)
    if (!p->u_desc || p->u_desc_cap < G) {
        cudaFree(p->u_desc);
        p->u_desc = nullptr;
        if (cudaMalloc(&p->u_desc, sizeof(UGraph) * (size_t)G) != cudaSuccess) {
            cudaGetLastError();
            return fail(ECL_SCC_ENOMEM, "batched graph table (%d graphs)", G);
        }
        p->u_desc_cap = G;
    }
    std::vector<UGraph> desc((size_t)G);
    {
        int64_t vo = 0, eo = 0, nmax = 1;
        for (int g = 0; g < G; g++) {
            desc[g] = UGraph{rp[g], ci[g], labels[g], nnz[g], eo, n[g], (int32_t)vo};
            nmax = std::max<int64_t>(nmax, std::max<int64_t>(n[g], nnz[g]));
            vo += n[g];
            eo += nnz[g];
        }
        CK(cudaMemcpyAsync(p->u_desc, desc.data(), sizeof(UGraph) * (size_t)G, cudaMemcpyHostToDevice, s));
        const int validate = !(p->flags & ECL_SCC_NO_VALIDATE);
        if (validate) CK(cudaMemsetAsync(&p->dc->err, 0, sizeof(int), s));
        const unsigned gx = (unsigned)std::max<int64_t>(1, std::min<int64_t>(cdiv(nmax, TPB), std::max(1, 148 * 16 / G)));
        p->launches++;
        k_union_all<<<dim3(gx, (unsigned)G), TPB, 0, s>>>((const UGraph*)p->u_desc, p->u_rp, p->u_ci, validate, &p->dc->err);
        if (validate) {
            CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
            CK(cudaStreamSynchronize(s));
            if (p->hc->err) return fail(ECL_SCC_ERANGE, "invalid CSR in batch");
        }
    }
    p->launches++; k_set1<<<1, 1, 0, s>>>(p->u_rp + N, (int32_t)M);
    CK(cudaGetLastError());
    const uint32_t saved = p->flags;
    p->flags |= ECL_SCC_NO_VALIDATE;
    int r = run_graph(p, (int32_t)N, M, p->u_rp, p->u_ci, p->u_lab, s, st, 0, nullptr, nullptr);
    p->flags = saved;
    if (r) return r;
    {
        int64_t nmax = 1;
        for (int g = 0; g < G; g++) nmax = std::max<int64_t>(nmax, n[g]);
        const unsigned gx = (unsigned)std::max<int64_t>(1, std::min<int64_t>(cdiv(nmax, TPB), std::max(1, 148 * 16 / G)));
        p->launches++; k_split_all<<<dim3(gx, (unsigned)G), TPB, 0, s>>>((const UGraph*)p->u_desc, p->u_lab);
    }
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(s));
    if (st) st->kernel_launches = p->launches;
    return ECL_SCC_OK;
}

// --------------------------------------------------------------------------- exchanges
int Exchange::allreduce(std::vector<int32_t*>& bufs, int64_t count, int op, cudaStream_t s) {
    cudaEvent_t a = nullptr, b = nullptr;
    if (ev) {
        if ((size_t)(2 * used + 2) > ev->size()) {
            for (int k = 0; k < 2; k++) {
                cudaEvent_t e;
                CK(cudaEventCreate(&e));
                ev->push_back(e);
            }
        }
        a = (*ev)[2 * used];
        b = (*ev)[2 * used + 1];
        used++;
        CK(cudaEventRecord(a, s));
    }
    if (int r = reduce(bufs, count, op, s)) return r;
    if (ev) CK(cudaEventRecord(b, s));
    bytes += 4 * count;
    return ECL_SCC_OK;
}
double Exchange::ms() const {
    double t = 0;
    for (int k = 0; ev && k < used; k++) {
        float x = 0.f;
        if (cudaEventElapsedTime(&x, (*ev)[2 * k], (*ev)[2 * k + 1]) == cudaSuccess) t += x;
        else cudaGetLastError();
    }
    return t;
}

// --------------------------------------------------------------------------- partitioned (halo) mode
HaloRank::~HaloRank() {
    plan_free(&p);
    cudaFree(lrp); cudaFree(lci); cudaFree(l2g); cudaFree(gmark); cudaFree(gidx); cudaFree(lab);
    cudaFree(hdeg); cudaFree(words);
    if (!hbuf_external) cudaFree(hbuf);
}

// workspace of one rank: rows [rb, re) of an n-vertex graph with at most m_cap local edges
// (the local graph has at most nloc + min(m_cap, n) vertices)
int halo_rank_alloc(HaloRank* R, int32_t n, int32_t rb, int32_t re, int64_t m_cap, uint32_t flags) {
    R->n = n; R->rb = rb; R->re = re; R->nloc = re - rb; R->m_cap = m_cap;
    const int64_t nl_max = std::min<int64_t>((int64_t)R->nloc + m_cap, n);
    if (flags & (ECL_SCC_TRIM2 | ECL_SCC_FOUR_SIG | ECL_SCC_COMPRESS | ECL_SCC_RAISE | ECL_SCC_CLUSTER))
        return fail(ECL_SCC_EUNSUPPORTED, "partitioned mode: Trim-2, the 4-signature variant, path compression and "
                                          "the P:190 variant are single-GPU only");
    R->p.flags = flags | ECL_SCC_NO_REORDER;       // the local -> global map is the storage map
    if (int r = plan_alloc(&R->p, (int32_t)std::max<int64_t>(nl_max, 1), std::max<int64_t>(m_cap, 1))) return r;
    const size_t n1 = (size_t)n + 1, nl1 = (size_t)nl_max + 1;
    cudaError_t e = cudaSuccess;
    auto A = [&](int32_t** ptr, size_t count) { if (e == cudaSuccess) e = cudaMalloc((void**)ptr, count * 4); };
    A(&R->p.hpos[0], nl1);
    A(&R->p.hpos[1], nl1);
    A(&R->lrp, nl1 + 1);
    A(&R->lci, (size_t)std::max<int64_t>(m_cap, 1));
    A(&R->l2g, nl1);
    A(&R->gmark, n1);
    A(&R->gidx, n1);
    A(&R->lab, n1);
    A(&R->words, 8);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ECL_SCC_ENOMEM, "partition workspace: %s", cudaGetErrorString(e));
    }
    R->p.lab_lo = rb;
    R->p.lab_hi = re;
    return ECL_SCC_OK;
}

// Rank r's local graph from its rows: ghosts, local -> global map, local CSR (halo.cuh)
static int halo_ingest(HaloRank& R, uint32_t flags, cudaStream_t s) {
    Plan* p = &R.p;
    const int32_t n = R.n;
    const unsigned gs = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
    CK(cudaMemsetAsync(R.gmark, 0, sizeof(int32_t) * (size_t)n, s));
    if (R.m) { p->launches++; k_halo_mark_ghosts<<<std::min<unsigned>(grid_for(R.m, TPB), 148 * 16), TPB, 0, s>>>(R.m, R.ci, R.rb, R.re, R.gmark); }
    if (int r = scan_excl<I1>(p, (const I1*)R.gmark, n, (I1*)R.gidx, (I1*)&p->dc->grand1, p->bsum, 0, s)) return r;
    int ng = 0;
    CK(cudaMemcpyAsync(&ng, &p->dc->grand1, sizeof(int), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    R.ng = ng;
    if ((int64_t)R.nloc + ng > p->n_cap) return fail(ECL_SCC_ECUDA, "internal: local graph exceeds its plan");
    p->launches += 2;
    k_halo_l2g<<<gs, TPB, 0, s>>>(n, R.rb, R.re, R.gmark, R.gidx, R.l2g);
    k_halo_local_csr<<<std::min<unsigned>(grid_for(std::max<int64_t>(R.m, R.nloc + ng + 1), TPB), 148 * 16), TPB, 0, s>>>(
        R.nloc, ng, R.m, R.rp, R.ci, R.rb, R.re, R.gidx, R.lrp, R.lci);
    CK(cudaGetLastError());
    (void)flags;
    return ECL_SCC_OK;
}

// The partitioned driver over this process's ranks R (1 with NCCL, P when emulated): the
// outer loop of run_graph per rank, in lockstep, with the halo exchanges (halo.cuh) at the
// points where the ranks must agree.
int run_halo(std::vector<HaloRank*>& R, Exchange& X, int32_t n, uint32_t flags, int32_t* labels, cudaStream_t s,
             ecl_scc_stats* st) {
    const int P = (int)R.size();
    if (st) memset(st, 0, sizeof(*st));
    const Prio Pr = make_prio((uint32_t)n, (flags & ECL_SCC_IDENTITY_IDS) != 0);
    const bool trim = !(flags & ECL_SCC_NO_TRIM);
    std::vector<int32_t*> bufs(P);
    auto each = [&](auto f) -> int {
        for (int r = 0; r < P; r++)
            if (int e = f(*R[r], r)) return e;
        return ECL_SCC_OK;
    };
    auto word_reduce = [&](int k, int op) -> int {   // all-reduce of device word k of every rank
        for (int r = 0; r < P; r++) bufs[r] = R[r]->words + k;
        return X.allreduce(bufs, 1, op, s);
    };
    auto read_word = [&](int k, int* out) -> int {
        CK(cudaMemcpyAsync(out, R[0]->words + k, sizeof(int), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        return ECL_SCC_OK;
    };
    int r = each([&](HaloRank& Q, int) -> int {
        Q.p.launches = 0;
        CK(cudaMemsetAsync(Q.words, 0, 8 * sizeof(int32_t), s));
        if (!(flags & ECL_SCC_NO_VALIDATE) && Q.nloc > 0) {
            Q.p.launches++;
            part::k_validate_part<<<std::min<unsigned>(grid_for(std::max<int64_t>(Q.nloc, Q.m), TPB), 148 * 16), TPB, 0, s>>>(
                Q.nloc, Q.m, Q.rp, Q.ci, n, Q.words + 2);
        }
        return ECL_SCC_OK;
    });
    if (r) return r;
    if ((r = word_reduce(2, 0))) return r;         // every rank learns of an invalid rank
    int err = 0;
    if ((r = read_word(2, &err))) return r;
    if (err) return fail(ECL_SCC_ERANGE, "partitioned: invalid local CSR on some rank");
    // ---- local graphs; the halo H = vertices that are a ghost on some rank
    if ((r = each([&](HaloRank& Q, int) { return halo_ingest(Q, flags, s); }))) return r;
    for (int q = 0; q < P; q++) bufs[q] = R[q]->gmark;
    if ((r = X.allreduce(bufs, n, 0, s))) return r;   // (ingest only: membership of all n IDs)
    int64_t H = 0;
    r = each([&](HaloRank& Q, int) -> int {
        Plan* p = &Q.p;
        const unsigned gs = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
        p->launches++; k_nonzero<<<gs, TPB, 0, s>>>(n, Q.gmark, Q.lab);          // (lab: scratch here)
        if (int e = scan_excl<I1>(p, (const I1*)Q.lab, n, (I1*)Q.gidx, (I1*)&p->dc->grand1, p->bsum, 0, s)) return e;
        int h = 0;
        CK(cudaMemcpyAsync(&h, &p->dc->grand1, sizeof(int), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        H = h;
        const int32_t nl = Q.nloc + Q.ng;
        p->launches++; k_halo_hpos<<<std::min<unsigned>(grid_for(std::max(nl, 1), TPB), 148 * 16), TPB, 0, s>>>(nl, Q.l2g, Q.gmark, Q.gidx, p->hpos[0]);
        p->launches++; k_fill<<<gs, TPB, 0, s>>>(n, Q.lab, INT32_MIN);
        CK(cudaGetLastError());
        return ECL_SCC_OK;
    });
    if (r) return r;
    if (R[0]->hcap < H || !R[0]->hbuf) {           // (grows once per plan; symmetric in NCCL mode)
        if ((r = X.halo_buffers(R, std::max<int64_t>(H, 1), s))) return r;
        for (HaloRank* Q : R) {
            cudaFree(Q->hdeg);
            if (cudaMalloc((void**)&Q->hdeg, sizeof(int32_t) * 2 * (size_t)std::max<int64_t>(H, 1)) != cudaSuccess) {
                cudaGetLastError();
                return fail(ECL_SCC_ENOMEM, "halo degree buffer");
            }
            Q->hcap = std::max<int64_t>(H, 1);
        }
    }
    const bool fused = R[0]->push.np > 0 || R[0]->push.mc;
    // ---- the single-GPU ingest of every local graph (CSC of the local rows)
    r = each([&](HaloRank& Q, int) -> int {
        Plan* p = &Q.p;
        Q.H = H;
        const int32_t nl = Q.nloc + Q.ng;
        if (int e = build_csc(p, nl, Q.m, Q.lrp, Q.lci, s)) return e;
        unsigned long long loc = 0;
        CK(cudaMemcpyAsync(&loc, &p->dc->local_e, sizeof(loc), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        p->low_locality = (double)loc < LOCAL_FP_LOCALITY * (double)std::max<int64_t>(Q.m, 1);
        p->orig_cur = Q.l2g;                        // local -> global: priorities and labels
        Q.g = WGraph{nullptr, Q.lrp, Q.lci, p->iptr[0], p->iadj[0], nl};
        Q.g.hpos = p->hpos[0];
        Q.ob = 1;
        return ECL_SCC_OK;
    });
    if (r) return r;
    int iters = 0;
    int64_t passes_total = 0;
    for (int iter = 1;; iter++) {
        if (iter > n + 2) return fail(ECL_SCC_ECUDA, "internal: partitioned outer loop exceeded n+2 iterations");
        // ---- Phase 3 (keep), the halo's kept degrees summed over the ranks, trim + compaction
        const int32_t* cin0 = nullptr;
        r = each([&](HaloRank& Q, int) {
            const int32_t* ci_ = iter == 1 ? cin0 : Q.p.cin[Q.ob ^ 1];
            const int32_t* co_ = iter == 1 ? cin0 : Q.p.cout[Q.ob ^ 1];
            return compaction(&Q.p, 0, iter, Q.g, ci_, co_, Q.ob, Q.lab, Pr, s);
        });
        if (r) return r;
        if (trim) {
            r = each([&](HaloRank& Q, int q) -> int {
                CK(cudaMemsetAsync(Q.hdeg, 0, sizeof(int32_t) * 2 * (size_t)H, s));
                if (Q.g.na) { Q.p.launches++; k_halo_deg_pack<<<std::min<unsigned>(grid_for(Q.g.na, TPB), 148 * 8), TPB, 0, s>>>(Q.g.na, Q.g.hpos, Q.p.kio, Q.hdeg); }
                bufs[q] = Q.hdeg;
                return ECL_SCC_OK;
            });
            if (r) return r;
            if ((r = X.allreduce(bufs, 2 * H, 1, s))) return r;
            r = each([&](HaloRank& Q, int) -> int {
                if (Q.g.na) { Q.p.launches++; k_halo_deg_apply<<<std::min<unsigned>(grid_for(Q.g.na, TPB), 148 * 8), TPB, 0, s>>>(Q.g.na, Q.g.hpos, Q.hdeg, Q.p.kio); }
                return ECL_SCC_OK;
            });
            if (r) return r;
        }
        int64_t live = 0;
        r = each([&](HaloRank& Q, int) -> int {
            Plan* p = &Q.p;
            const int32_t* ci_ = iter == 1 ? nullptr : p->cin[Q.ob ^ 1];
            const int32_t* co_ = iter == 1 ? nullptr : p->cout[Q.ob ^ 1];
            if (int e = compaction(p, 1, iter, Q.g, ci_, co_, Q.ob, Q.lab, Pr, s)) return e;
            CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
            CK(cudaStreamSynchronize(s));
            if (p->hc->err == 3) return fail(ECL_SCC_ECUDA, "internal: asynchronous Phase 2 stalled (watchdog)");
            const int4 t = p->hc->totals;
            if (t.y != t.z) return fail(ECL_SCC_ECUDA, "internal: CSR/CSC survivor mismatch %d vs %d", t.y, t.z);
            p->nchunks_cur = p->hc->nchunks;
            Q.g = WGraph{p->act[Q.ob], p->optr[Q.ob], p->oadj[Q.ob], p->iptr[Q.ob], p->iadj[Q.ob], t.x};
            Q.g.hpos = p->hpos[Q.ob];
            live += t.y;
            // the exchange buffer restarts with every Phase 2 (before the barrier below, so no
            // rank can push into a buffer that is still to be cleared)
            CK(cudaMemsetAsync(Q.hbuf, 0, sizeof(int32_t) * 2 * (size_t)H, s));
            const int ty = t.y;
            CK(cudaMemcpyAsync(Q.words + 1, &ty, sizeof(int), cudaMemcpyHostToDevice, s));
            return ECL_SCC_OK;
        });
        if (r) return r;
        if ((r = word_reduce(1, 1))) return r;      // live edges of all ranks (termination)
        int glive = 0;
        if ((r = read_word(1, &glive))) return r;
        if (st && iter - 1 < ECL_SCC_TRACE_MAX) st->edges_in[iter - 1] = glive;
        if (glive == 0) {
            // every remaining vertex is unfinished and edgeless on every rank: a singleton
            r = each([&](HaloRank& Q, int) -> int {
                if (Q.g.na) { Q.p.launches++; k_halo_final<<<std::min<unsigned>(grid_for(Q.g.na, TPB), 148 * 8), TPB, 0, s>>>(Q.g.na, Q.g.act, Q.l2g, Q.rb, Q.re, Q.lab); }
                return ECL_SCC_OK;
            });
            if (r) return r;
            if (st && iter - 1 < ECL_SCC_TRACE_MAX) st->edges_in[iter - 1] = 0;
            break;
        }
        if (st && iter >= 2 && iter - 2 < ECL_SCC_TRACE_MAX) st->edges_kept[iter - 2] = glive;
        // ---- Phase 2: local fixed points; raised halo copies pushed to every rank; fold in
        int64_t rounds = 0;
        for (int round = 0;; round++) {
            r = each([&](HaloRank& Q, int) -> int {
                Plan* p = &Q.p;
                HaloPush push = Q.push;
                push.hpos = Q.g.hpos;
                if (!fused) {                         // NCCL all-reduce exchange: own buffer only
                    push.np = 1;
                    push.peer[0] = Q.hbuf;
                    push.mc = nullptr;
                    push.sys = 0;
                }
                int64_t passes = 0;
                if (Q.g.na == 0) return ECL_SCC_OK;
                if (int e = propagate(p, Q.g, p->cin[Q.ob], p->cout[Q.ob], p->nchunks_cur, s, &passes, false, &push,
                                      round > 0))
                    return e;
                if (!fused && pack_path(p, p->nchunks_cur) && !(flags & ECL_SCC_NO_ASYNC)) {
                    // (asynchronous kernel pushed its raises into the own buffer already)
                }
                return ECL_SCC_OK;
            });
            if (r) return r;
            rounds++;
            if (!fused) {
                for (int q = 0; q < P; q++) bufs[q] = R[q]->hbuf;
                if ((r = X.allreduce(bufs, 2 * H, 0, s))) return r;
            } else if ((r = word_reduce(0, 0))) {     // barrier: every rank's pushes have landed
                return r;
            }
            r = each([&](HaloRank& Q, int) -> int {
                Plan* p = &Q.p;
                CK(cudaMemsetAsync(Q.words, 0, sizeof(int32_t), s));
                if (Q.g.na == 0) return ECL_SCC_OK;
                const bool async = pack_path(p, p->nchunks_cur) && !(flags & ECL_SCC_NO_ASYNC);
                const bool dirty = !async && p->nchunks_cur == 0 && !(flags & (ECL_SCC_SYNC_PASSES | ECL_SCC_NO_DIRTY));
                p->launches++;
                k_halo_apply<<<std::min<unsigned>(grid_for(Q.g.na, TPB), 148 * 8), TPB, 0, s>>>(
                    Q.g, Q.hbuf, p->cin[Q.ob], p->cout[Q.ob], async ? p->aq_state : nullptr,
                    async ? p->aq_seen : nullptr, async ? p->aq_ctr + AQ_PEND : nullptr, dirty ? p->dirty : nullptr, TILE,
                    Q.words);
                CK(cudaGetLastError());
                return ECL_SCC_OK;
            });
            if (r) return r;
            if ((r = word_reduce(0, 0))) return r;  // did any rank take a larger copy?
            int inj = 0;
            if ((r = read_word(0, &inj))) return r;
            if (!inj) break;
            if (round > 4 * n + 64) return fail(ECL_SCC_ECUDA, "internal: halo exchange did not converge");
        }
        iters = iter;
        passes_total += rounds;
        if (st && iter - 1 < ECL_SCC_TRACE_MAX) st->passes_iter[iter - 1] = rounds;
        for (HaloRank* Q : R) Q->ob ^= 1;
    }
    // ---- labels: the owners' entries, combined; priorities -> max vertex IDs (k_relabel_*)
    for (int q = 0; q < P; q++) bufs[q] = R[q]->lab;
    if ((r = X.allreduce(bufs, n, 0, s))) return r;
    HaloRank& Q = *R[0];
    const unsigned gr = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
    if (!Pr.ids) {
        Q.p.launches += 2;
        CK(cudaMemsetAsync(Q.gidx, 0xFF, sizeof(int32_t) * (size_t)n, s));
        k_relabel_fold<<<gr, TPB, 0, s>>>(n, Q.lab, Q.gidx);
        k_relabel_apply<<<gr, TPB, 0, s>>>(n, Q.lab, Q.gidx);
    }
    CK(cudaMemcpyAsync(labels, Q.lab, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToDevice, s));
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(s));
    if (st) {
        int64_t launches = 0, vv = 0, ve = 0;
        for (HaloRank* q : R) {
            launches += q->p.launches;
            CK(cudaMemcpy(q->p.hc, q->p.dc, sizeof(DevCounters), cudaMemcpyDeviceToHost));
            vv += (int64_t)q->p.hc->visit_v;
            ve += (int64_t)q->p.hc->visit_e;
        }
        st->iterations = iters;
        st->trace_len = std::min(iters, ECL_SCC_TRACE_MAX);
        st->passes = passes_total;
        st->kernel_launches = launches;
        st->prop_bytes = 20 * vv + 12 * ve;
        st->ms_comm = X.ms();
        st->comm_bytes = X.bytes;
        st->exchanges = X.used;
    }
    return ECL_SCC_OK;
}

// Sweep levels of the SCC condensation (levels.cuh); plan buffers serve as workspace.
// f4, tile mode (levels.cuh k_lk_*), after k_lv_count filled msize / odeg: *used = 0 means
// "Kahn's rounds instead" (cross edges mostly between tiles, or a node with a long cross-edge
// list, which one lane would walk)
static int run_levels_tiles(Plan* p, int32_t n, const int32_t* rp, const int32_t* ci, const int32_t* lab,
                            int32_t* out, int32_t* depth, cudaStream_t s, int* used) {
    *used = 0;
    LvCtl* ctl = (LvCtl*)p->lv_ctl;
    const int32_t* msize = p->kout;
    int32_t* odeg = p->act[1];
    int32_t* cptr = p->optr[1];
    int32_t* cadj = p->oadj[1];
    int32_t* ccur = p->iptr[1];                     // (Kahn's rounds use newidx as their cursor)
    int32_t* icnt = p->cin[1];
    int32_t* ecnt = p->cout[1];
    int32_t* lvl = p->cin[0];
    int32_t* lvl_ext = p->cout[0];
    const size_t nb = sizeof(int32_t) * (size_t)n;
    const unsigned gs = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
    if (int r = scan_excl<I1>(p, (const I1*)odeg, n, (I1*)cptr, (I1*)&p->dc->grand1, p->bsum, 1, s)) return r;
    CK(cudaMemsetAsync(ccur, 0, nb, s));
    CK(cudaMemsetAsync(icnt, 0, nb, s));
    CK(cudaMemsetAsync(ecnt, 0, nb, s));
    p->launches++; k_lk_fill<<<gs, TPB, 0, s>>>(n, rp, ci, lab, cptr, ccur, cadj, icnt, ecnt);
    p->launches++; k_lk_init<<<gs, TPB, 0, s>>>(n, msize, cptr, icnt, lvl, lvl_ext, ctl);
    CK(cudaGetLastError());
    LvCtl h;
    CK(cudaMemcpyAsync(&h, ctl, sizeof(LvCtl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (h.maxodeg > 256) {
        CK(cudaMemsetAsync(ctl, 0, sizeof(LvCtl), s));     // Kahn's rounds count the SCCs again
        return ECL_SCC_OK;
    }
    *used = 1;
    if (int r = ensure_async(p)) return r;
    if (!p->lk_resident) {
        CK(cudaFuncSetAttribute(k_lk_run, cudaFuncAttributeMaxDynamicSharedMemorySize, LK_ECAP * 4));
        CK(cudaFuncSetAttribute(k_lk_run, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared));
        int per_sm = 0, sms = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_lk_run, LK_TH, LK_ECAP * 4));
        CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device));
        p->lk_resident = (int64_t)std::max(1, per_sm) * sms;
    }
    const unsigned ntiles = (unsigned)cdiv(n, LK_TT);
    AsyncQ Q{p->aq_state, p->aq_seen, p->aq_ctr};
    const int claim = (int)std::min<int64_t>(16, std::max<int64_t>(1, ntiles / p->lk_resident));
    CK(cudaMemsetAsync(&p->dc->err, 0, sizeof(int), s));
    CK(cudaMemsetAsync(&p->dc->passes, 0, sizeof(unsigned long long), s));
    CK(cudaMemsetAsync(&p->dc->prof[0], 0, sizeof(unsigned long long), s));
    p->launches++; k_async_init<<<grid_for((int64_t)ntiles, TPB), TPB, 0, s>>>(Q, (int)ntiles);
    const LkState L{cptr, cadj, icnt, ecnt, lvl, lvl_ext, n};
    p->launches++;
    k_lk_run<<<(unsigned)std::min<int64_t>(ntiles, p->lk_resident), LK_TH, LK_ECAP * 4, s>>>(L, p->dc, Q, claim);
    p->launches++; k_lk_apply<<<gs, TPB, 0, s>>>(n, lab, msize, icnt, lvl, out, ctl);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(&h, ctl, sizeof(LvCtl), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(p->hc, p->dc, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (getenv("ECL_SCC_DEBUG"))
        fprintf(stderr, "[ecl_scc] levels (tiles): %d SCCs, cross edges %llu inside tiles / %llu between, "
                        "%.2f visits per tile (%.2f found nothing ready)\n", h.nscc, h.intra, h.cross,
                (double)p->hc->passes / ntiles, (double)p->hc->prof[0] / ntiles);
    if (p->hc->err) return fail(ECL_SCC_ECUDA, "levels: the tile queue stalled (error %d)", p->hc->err);
    if (h.reached != h.nscc)
        return fail(ECL_SCC_ERANGE, "levels: the labels induce a cyclic condensation (%d of %d SCCs reached)",
                    h.reached, h.nscc);
    if (depth) *depth = h.depth;
    return ECL_SCC_OK;
}

int run_levels(Plan* p, int32_t n, const int32_t* rp, const int32_t* ci, const int32_t* lab, int32_t* out,
               int32_t* depth, cudaStream_t s) {
    if (!p->lv_ctl) {
        cudaError_t e = cudaMalloc(&p->lv_ctl, sizeof(LvCtl));
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(ECL_SCC_ENOMEM, "levels control block: %s", cudaGetErrorString(e));
        }
        int per_sm = 0, dev = 0, sms = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_lv_run, 512, 0));
        CK(cudaGetDevice(&dev));
        CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        // one CTA per SM: the round barrier's cost grows with the CTAs that arrive at it
        p->lv_resident = std::max(1, std::min(per_sm, 1)) * sms;
        if (p->knob_lv_ctas) p->lv_resident = std::min(p->lv_resident, p->knob_lv_ctas);   // tuning knob
    }
    LvCtl* ctl = (LvCtl*)p->lv_ctl;
    int32_t* indeg = p->kin;
    int32_t* msize = p->kout;
    int32_t* mptr = p->optr[0];
    int32_t* cursor = p->newidx;
    int32_t* memb = p->act[0];
    int32_t* lvl = p->cin[0];
    int2* qa = p->cnt;
    int2* qb = (int2*)p->emask;
    const size_t nb = sizeof(int32_t) * (size_t)n;
    CK(cudaMemsetAsync(indeg, 0, nb, s));
    CK(cudaMemsetAsync(msize, 0, nb, s));
    CK(cudaMemsetAsync(cursor, 0, nb, s));
    CK(cudaMemsetAsync(ctl, 0, sizeof(LvCtl), s));
    const unsigned gs = std::min<unsigned>(grid_for(n, TPB), 148 * 16);
    const bool tiles = !(p->flags & ECL_SCC_NO_ASYNC);
    int32_t* odeg = tiles ? p->act[1] : nullptr;
    if (tiles) CK(cudaMemsetAsync(odeg, 0, nb, s));
    p->launches++; k_lv_count<<<gs, TPB, 0, s>>>(n, rp, ci, lab, indeg, msize, &ctl->err, odeg, &ctl->intra);
    CK(cudaGetLastError());
    LvCtl h0;
    {   // every later kernel indexes by label: reject labels outside [0, n) before them
        CK(cudaMemcpyAsync(&h0, ctl, sizeof(LvCtl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (h0.err) return fail(ECL_SCC_ERANGE, "levels: a label lies outside [0, n)");
    }
    // the tile mode pays when the cross edges mostly stay inside tiles (meshes: ~0.9; R-MAT: ~0)
    if (tiles && (double)h0.intra >= 0.5 * (double)(h0.intra + h0.cross)) {
        int used = 0;
        if (int r = run_levels_tiles(p, n, rp, ci, lab, out, depth, s, &used)) return r;
        if (used) return ECL_SCC_OK;
    }
    int r = scan_excl<I1>(p, (const I1*)msize, n, (I1*)mptr, (I1*)&p->dc->grand1, p->bsum, 1, s);
    if (r) return r;
    p->launches++; k_lv_fill<<<gs, TPB, 0, s>>>(n, lab, mptr, cursor, memb);
    p->launches++; k_lv_init<<<gs, TPB, 0, s>>>(n, indeg, msize, mptr, lvl, qa, ctl);
    CK(cudaGetLastError());
    void* args[] = {(void*)&rp, (void*)&ci, (void*)&lab, &mptr, &memb, &indeg, &lvl, &qa, &qb, &ctl};
    p->launches++;
    CK(cudaLaunchCooperativeKernel((const void*)k_lv_run, dim3(p->lv_resident), dim3(512), args, 0, s));
    p->launches++; k_lv_apply<<<gs, TPB, 0, s>>>(n, lab, lvl, out);
    CK(cudaGetLastError());
    LvCtl h;
    CK(cudaMemcpyAsync(&h, ctl, sizeof(LvCtl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (h.err) return fail(ECL_SCC_ERANGE, "levels: a label lies outside [0, n)");
    if (h.reached != h.nscc)
        return fail(ECL_SCC_ERANGE, "levels: the labels induce a cyclic condensation (%d of %d SCCs reached)",
                    h.reached, h.nscc);
    if (depth) *depth = h.depth;
    return ECL_SCC_OK;
}

}  // namespace eclscc

// =========================================================================== C ABI
using namespace eclscc;

struct ecl_scc_plan_s {
    Plan p;
};

static int check_graph_args(int32_t n, int64_t nnz, const void* rp, const void* ci, const void* out) {
    if (n < 0 || nnz < 0) return fail(ECL_SCC_EINVAL, "negative size (n=%d, nnz=%lld)", n, (long long)nnz);
    if (n > 0 && (!rp || !out)) return fail(ECL_SCC_EINVAL, "NULL row_ptr or labels_out");
    if (nnz > 0 && !ci) return fail(ECL_SCC_EINVAL, "NULL col_idx");
    if (nnz >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "nnz >= 2^31 needs 64-bit offsets");
    if (n == INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "n must be < 2^31 - 1");
    return ECL_SCC_OK;
}

extern "C" {

int ecl_scc_version(void) { return 100; }

const char* ecl_scc_status_string(int s) {
    switch (s) {
        case ECL_SCC_OK: return "ok";
        case ECL_SCC_EINVAL: return "invalid argument";
        case ECL_SCC_ERANGE: return "malformed graph (offsets or column out of range)";
        case ECL_SCC_ENOMEM: return "out of device memory";
        case ECL_SCC_ECUDA: return "CUDA error";
        case ECL_SCC_ENCCL: return "NCCL error";
        case ECL_SCC_EUNSUPPORTED: return "unsupported";
        default: return "unknown status";
    }
}

const char* ecl_scc_last_error(void) { return last_err(); }

int ecl_scc_plan_create(int32_t n_max, int64_t nnz_max, uint32_t flags, ecl_scc_plan_t* out) {
    clear_err();
    if (!out || n_max < 0 || nnz_max < 0) return fail(ECL_SCC_EINVAL, "plan_create: bad arguments");
    if (nnz_max >= (int64_t)INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "nnz_max >= 2^31");
    ecl_scc_plan_s* h = (ecl_scc_plan_s*)calloc(1, sizeof(ecl_scc_plan_s));
    if (!h) return fail(ECL_SCC_ENOMEM, "host allocation");
    if ((flags & (ECL_SCC_COMPRESS | ECL_SCC_RAISE)) && (flags & (ECL_SCC_FOUR_SIG | ECL_SCC_CLUSTER))) {
        free(h);
        return fail(ECL_SCC_EINVAL, "plan_create: ECL_SCC_COMPRESS / ECL_SCC_RAISE apply to the two-signature, "
                                    "single-CTA-tile method");
    }
    if ((flags & ECL_SCC_TRIM2) && (flags & ECL_SCC_NO_TRIM)) {
        free(h);
        return fail(ECL_SCC_EINVAL, "plan_create: ECL_SCC_TRIM2 runs with Trim-1 (not with ECL_SCC_NO_TRIM)");
    }
    h->p.flags = flags;
    int r = plan_alloc(&h->p, n_max, nnz_max);
    if (r) {
        plan_free(&h->p);
        free(h);
        return r;
    }
    *out = h;
    return ECL_SCC_OK;
}

int ecl_scc_plan_counters(ecl_scc_plan_t plan, uint64_t out[8]) {
    clear_err();
    if (!plan || !out) return fail(ECL_SCC_EINVAL, "plan_counters: bad arguments");
    CK(cudaMemcpy(out, plan->p.dc->prof, sizeof(plan->p.dc->prof), cudaMemcpyDeviceToHost));
    return ECL_SCC_OK;
}

int ecl_scc_plan_destroy(ecl_scc_plan_t plan) {
    clear_err();
    if (!plan) return ECL_SCC_OK;
    plan_free(&plan->p);
    free(plan);
    return ECL_SCC_OK;
}

int ecl_scc_async(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx, int32_t* labels_out,
                  ecl_scc_stream_t stream, ecl_scc_plan_t plan, ecl_scc_stats* stats) {
    clear_err();
    int r = check_graph_args(n, nnz, row_ptr, col_idx, labels_out);
    if (r) return r;
    if (stats) memset(stats, 0, sizeof(*stats));
    if (n == 0) return ECL_SCC_OK;
    if (plan && (plan->p.n_cap < n || plan->p.m_cap < nnz))
        return fail(ECL_SCC_EINVAL, "plan too small (n_max=%d, nnz_max=%lld)", plan->p.n_cap, (long long)plan->p.m_cap);
    ecl_scc_plan_t tmp = nullptr;
    if (!plan) {
        r = ecl_scc_plan_create(n, nnz, 0, &tmp);
        if (r) return r;
        plan = tmp;
    }
    plan->p.launches = 0;
    r = run_graph(&plan->p, n, nnz, row_ptr, col_idx, labels_out, (cudaStream_t)stream, stats, 0, nullptr, nullptr);
    if (tmp) ecl_scc_plan_destroy(tmp);
    return r;
}

int ecl_scc_host(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx, int32_t* labels_out,
                 ecl_scc_stream_t stream, ecl_scc_plan_t plan, ecl_scc_stats* stats) {
    clear_err();
    int r = check_graph_args(n, nnz, row_ptr, col_idx, labels_out);
    if (r) return r;
    if (stats) memset(stats, 0, sizeof(*stats));
    if (n == 0) return ECL_SCC_OK;
    if (plan && (plan->p.n_cap < n || plan->p.m_cap < nnz))
        return fail(ECL_SCC_EINVAL, "plan too small (n_max=%d, nnz_max=%lld)", plan->p.n_cap, (long long)plan->p.m_cap);
    ecl_scc_plan_t tmp = nullptr;
    if (!plan) {
        r = ecl_scc_plan_create(n, nnz, 0, &tmp);
        if (r) return r;
        plan = tmp;
    }
    Plan* p = &plan->p;
    cudaStream_t s = (cudaStream_t)stream;
    if (!p->h_rp || p->h_n_cap < n || p->h_m_cap < nnz) {          // device copies, sized for the plan
        cudaFree(p->h_rp); cudaFree(p->h_ci); cudaFree(p->h_lab);
        p->h_rp = p->h_ci = p->h_lab = nullptr;
        cudaError_t e = cudaMalloc((void**)&p->h_rp, sizeof(int32_t) * ((size_t)p->n_cap + 1));
        if (e == cudaSuccess) e = cudaMalloc((void**)&p->h_ci, sizeof(int32_t) * (size_t)std::max<int64_t>(p->m_cap, 1));
        if (e == cudaSuccess) e = cudaMalloc((void**)&p->h_lab, sizeof(int32_t) * ((size_t)p->n_cap + 1));
        if (e != cudaSuccess) {
            cudaGetLastError();
            if (tmp) ecl_scc_plan_destroy(tmp);
            return fail(ECL_SCC_ENOMEM, "host-buffer staging: %s", cudaGetErrorString(e));
        }
        p->h_n_cap = p->n_cap;
        p->h_m_cap = p->m_cap;
    }
    p->launches = 0;
    cudaError_t e = cudaMemcpyAsync(p->h_rp, row_ptr, sizeof(int32_t) * ((size_t)n + 1), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && nnz)
        e = cudaMemcpyAsync(p->h_ci, col_idx, sizeof(int32_t) * (size_t)nnz, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) r = fail(ECL_SCC_ECUDA, "host-to-device copy: %s", cudaGetErrorString(e));
    if (!r) r = run_graph(p, n, nnz, p->h_rp, p->h_ci, p->h_lab, s, stats, 0, nullptr, nullptr);
    if (!r) {
        e = cudaMemcpyAsync(labels_out, p->h_lab, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) r = fail(ECL_SCC_ECUDA, "device-to-host copy: %s", cudaGetErrorString(e));
    }
    if (tmp) ecl_scc_plan_destroy(tmp);
    return r;
}

int ecl_scc(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx, int32_t* labels_out) {
    return ecl_scc_async(n, nnz, row_ptr, col_idx, labels_out, nullptr, nullptr, nullptr);
}

int ecl_scc_debug_run(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx, uint32_t flags,
                      int32_t stop_iter, int32_t* sig_in, int32_t* sig_out, ecl_scc_stream_t stream,
                      ecl_scc_stats* stats) {
    clear_err();
    int r = check_graph_args(n, nnz, row_ptr, col_idx, sig_in);
    if (r) return r;
    if (stop_iter < 1 || (n > 0 && !sig_out)) return fail(ECL_SCC_EINVAL, "debug_run: stop_iter >= 1 and sig_out required");
    if (n == 0) return ECL_SCC_OK;
    ecl_scc_plan_t tmp = nullptr;
    r = ecl_scc_plan_create(n, nnz, flags, &tmp);
    if (r) return r;
    int32_t* lab = nullptr;
    if (cudaMalloc((void**)&lab, sizeof(int32_t) * (size_t)n) != cudaSuccess) {
        cudaGetLastError();
        ecl_scc_plan_destroy(tmp);
        return fail(ECL_SCC_ENOMEM, "debug_run labels");
    }
    r = run_graph(&tmp->p, n, nnz, row_ptr, col_idx, lab, (cudaStream_t)stream, stats, stop_iter, sig_in, sig_out);
    cudaStreamSynchronize((cudaStream_t)stream);
    cudaFree(lab);
    cudaStreamSynchronize((cudaStream_t)stream);
    ecl_scc_plan_destroy(tmp);
    return r;
}

int ecl_scc_batched(int32_t G, const int32_t* n, const int64_t* nnz, const int32_t* const* row_ptr,
                    const int32_t* const* col_idx, int32_t* const* labels_out, ecl_scc_stream_t stream,
                    ecl_scc_plan_t plan, ecl_scc_stats* stats) {
    clear_err();
    if (G < 0 || (G > 0 && (!n || !nnz || !row_ptr || !col_idx || !labels_out)))
        return fail(ECL_SCC_EINVAL, "batched: bad arguments");
    int64_t N = 0, M = 0;
    for (int g = 0; g < G; g++) {
        int r = check_graph_args(n[g], nnz[g], row_ptr[g], col_idx[g], labels_out[g]);
        if (r) return r;
        N += n[g];
        M += nnz[g];
    }
    if (stats) memset(stats, 0, sizeof(*stats));
    if (N == 0) return ECL_SCC_OK;
    if (N >= INT32_MAX || M >= INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "batch union exceeds 2^31 vertices or edges");
    if (plan && (plan->p.n_cap < N || plan->p.m_cap < M))
        return fail(ECL_SCC_EINVAL, "plan too small for the batch union");
    ecl_scc_plan_t tmp = nullptr;
    if (!plan) {
        int r = ecl_scc_plan_create((int32_t)N, M, 0, &tmp);
        if (r) return r;
        plan = tmp;
    }
    int r = run_batched(&plan->p, G, n, nnz, row_ptr, col_idx, labels_out, (cudaStream_t)stream, stats);
    if (tmp) ecl_scc_plan_destroy(tmp);
    return r;
}

int ecl_scc_batched_host(int32_t G, const int32_t* n, const int64_t* nnz, const int32_t* const* row_ptr,
                         const int32_t* const* col_idx, int32_t* const* labels_out, ecl_scc_stream_t stream,
                         ecl_scc_plan_t plan, ecl_scc_stats* stats) {
    clear_err();
    if (G < 0 || (G > 0 && (!n || !nnz || !row_ptr || !col_idx || !labels_out)))
        return fail(ECL_SCC_EINVAL, "batched_host: bad arguments");
    int64_t N = 0, M = 0;
    for (int g = 0; g < G; g++) {
        int r = check_graph_args(n[g], nnz[g], row_ptr[g], col_idx[g], labels_out[g]);
        if (r) return r;
        N += n[g];
        M += nnz[g];
    }
    if (stats) memset(stats, 0, sizeof(*stats));
    if (N == 0) return ECL_SCC_OK;
    if (N >= INT32_MAX || M >= INT32_MAX) return fail(ECL_SCC_EUNSUPPORTED, "batch union exceeds 2^31 vertices or edges");
    if (plan && (plan->p.n_cap < N || plan->p.m_cap < M))
        return fail(ECL_SCC_EINVAL, "plan too small for the batch union");
    ecl_scc_plan_t tmp = nullptr;
    if (!plan) {
        int r = ecl_scc_plan_create((int32_t)N, M, 0, &tmp);
        if (r) return r;
        plan = tmp;
    }
    Plan* p = &plan->p;
    cudaStream_t s = (cudaStream_t)stream;
    // device staging of the whole batch (graph g at offsets sum_{h<g} (n_h + 1), sum nnz_h, sum n_h)
    const int64_t rp_need = N + G, ci_need = std::max<int64_t>(M, 1), lab_need = N;
    cudaError_t e = cudaSuccess;
    if (p->hb_rp_cap < rp_need) {
        cudaFree(p->hb_rp); p->hb_rp = nullptr; p->hb_rp_cap = 0;
        e = cudaMalloc((void**)&p->hb_rp, sizeof(int32_t) * (size_t)rp_need);
        if (e == cudaSuccess) p->hb_rp_cap = rp_need;
    }
    if (e == cudaSuccess && p->hb_ci_cap < ci_need) {
        cudaFree(p->hb_ci); p->hb_ci = nullptr; p->hb_ci_cap = 0;
        e = cudaMalloc((void**)&p->hb_ci, sizeof(int32_t) * (size_t)ci_need);
        if (e == cudaSuccess) p->hb_ci_cap = ci_need;
    }
    if (e == cudaSuccess && p->hb_lab_cap < lab_need) {
        cudaFree(p->hb_lab); p->hb_lab = nullptr; p->hb_lab_cap = 0;
        e = cudaMalloc((void**)&p->hb_lab, sizeof(int32_t) * (size_t)lab_need);
        if (e == cudaSuccess) p->hb_lab_cap = lab_need;
    }
    if (e != cudaSuccess) {
        cudaGetLastError();
        if (tmp) ecl_scc_plan_destroy(tmp);
        return fail(ECL_SCC_ENOMEM, "batch host-buffer staging: %s", cudaGetErrorString(e));
    }
    std::vector<const int32_t*> drp(G), dci(G);
    std::vector<int32_t*> dlab(G);
    int64_t ro = 0, co = 0, lo = 0;
    for (int g = 0; g < G && e == cudaSuccess; g++) {
        drp[g] = p->hb_rp + ro;
        dci[g] = nnz[g] ? p->hb_ci + co : nullptr;
        dlab[g] = n[g] ? p->hb_lab + lo : nullptr;
        e = cudaMemcpyAsync(p->hb_rp + ro, row_ptr[g], sizeof(int32_t) * ((size_t)n[g] + 1), cudaMemcpyHostToDevice, s);
        if (e == cudaSuccess && nnz[g])
            e = cudaMemcpyAsync(p->hb_ci + co, col_idx[g], sizeof(int32_t) * (size_t)nnz[g], cudaMemcpyHostToDevice, s);
        ro += n[g] + 1;
        co += nnz[g];
        lo += n[g];
    }
    int r = e == cudaSuccess ? ECL_SCC_OK : fail(ECL_SCC_ECUDA, "host-to-device copy: %s", cudaGetErrorString(e));
    if (!r) r = run_batched(p, G, n, nnz, drp.data(), dci.data(), dlab.data(), s, stats);
    for (int g = 0; g < G && !r; g++) {
        if (!n[g]) continue;
        e = cudaMemcpyAsync(labels_out[g], dlab[g], sizeof(int32_t) * (size_t)n[g], cudaMemcpyDeviceToHost, s);
        if (e != cudaSuccess) r = fail(ECL_SCC_ECUDA, "device-to-host copy: %s", cudaGetErrorString(e));
    }
    if (!r && (e = cudaStreamSynchronize(s)) != cudaSuccess) r = fail(ECL_SCC_ECUDA, "device-to-host copy: %s", cudaGetErrorString(e));
    if (tmp) ecl_scc_plan_destroy(tmp);
    return r;
}

int ecl_scc_levels(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx, const int32_t* labels,
                   int32_t* levels_out, int32_t* depth_out, ecl_scc_stream_t stream, ecl_scc_plan_t plan) {
    clear_err();
    int r = check_graph_args(n, nnz, row_ptr, col_idx, levels_out);
    if (r) return r;
    if (n > 0 && !labels) return fail(ECL_SCC_EINVAL, "levels: NULL labels");
    if (depth_out) *depth_out = 0;
    if (n == 0) return ECL_SCC_OK;
    if (plan && plan->p.n_cap < n) return fail(ECL_SCC_EINVAL, "plan too small (n_max=%d)", plan->p.n_cap);
    ecl_scc_plan_t tmp = nullptr;
    if (!plan) {
        r = ecl_scc_plan_create(n, nnz, 0, &tmp);
        if (r) return r;
        plan = tmp;
    }
    plan->p.launches = 0;
    r = run_levels(&plan->p, n, row_ptr, col_idx, labels, levels_out, depth_out, (cudaStream_t)stream);
    if (tmp) ecl_scc_plan_destroy(tmp);
    return r;
}

int ecl_scc_partition_rows(int32_t P, int32_t n, const int32_t* rp, int32_t* bounds) {
    clear_err();
    if (P < 1 || n < 0 || !rp || !bounds) return fail(ECL_SCC_EINVAL, "partition_rows: bad arguments");
    const int64_t m = rp[n];
    bounds[0] = 0;
    for (int r = 1; r < P; r++) {
        // first row whose start offset reaches r*m/P
        const int64_t target = (m * r + P - 1) / P;
        int32_t lo = bounds[r - 1], hi = n;
        while (lo < hi) {
            const int32_t mid = lo + (hi - lo) / 2;
            if ((int64_t)rp[mid] < target) lo = mid + 1; else hi = mid;
        }
        bounds[r] = lo;
    }
    bounds[P] = n;
    return ECL_SCC_OK;
}

}  // extern "C"
