// tail.cuh -- the last outer iterations of Alg. 1 in ONE persistent launch.
//
// After a few outer iterations the working graph is small (C4: 27k vertices at iteration 9,
// 8 left at 14), and every further iteration costs ~90 us of launches and host round trips
// for microseconds of work: the compaction kernels, the tile pack, the Phase-2 launch and
// two stream synchronisations.  Once the compacted graph is below the tail threshold (and
// has no long rows), k_tail runs every remaining iteration on the device with grid
// barriers and no compaction at all:
//   Phase 2 (Alg. 1 l.7-14)   passes of owner-computes pulls in place (each vertex
//                             writes only its own v_in / v_out: no atomics), alternating
//                             ascending / descending over contiguous vertex ranges, until
//                             a pass changes nothing (that pass saw a consistent state:
//                             the fixed point, reading 12)
//   Phase 3 (l.15-19)  an edge entry whose ends carry different (v_in, v_out) pairs,
//                             or whose pair is finished, is cleared to -1 in place (CSR
//                             and CSC entries decide independently with the same rule)
//   Trim-1             one simultaneous round on the kept degrees
//   Phase 1 (l.3-6, R2)       survivors restart from their priority; a vertex without
//                             live edges leaves with its label (as k_compact_map)
// until no live edge is left.  Labels and per-iteration trace (edges entering Phase 2,
// vertices, kept edges) equal the compacting path's (same rules, reading 12); pass
// counts are schedule dependent.
#pragma once
#include "common.cuh"

namespace eclscc {

constexpr int TAIL_TH = 512;

struct TailTrace {                       // per absolute outer iteration k (index k-1)
    long long edges_in[ECL_SCC_TRACE_MAX];
    long long vertices_in[ECL_SCC_TRACE_MAX];
    long long edges_kept[ECL_SCC_TRACE_MAX];
    long long passes[ECL_SCC_TRACE_MAX];
    int last_iter;                       // last iteration that ran Phase 2
    int err;
    unsigned bar[2];                     // grid barrier: arrivals, generation
    int flag[3];                         // per-pass "changed" words (pass % 3)
    long long cnt[4][3];                 // per-iteration (iter % 4): kept, edges, vertices
};

// grid barrier among the co-resident CTAs of a cooperative launch (one CTA: a block barrier)
__device__ __forceinline__ void tail_bar(unsigned* bar, int G) {
    __syncthreads();
    if (G == 1) return;
    if (threadIdx.x == 0) {
        volatile unsigned* vb = bar;
        const unsigned gen = vb[1];
        __threadfence();
        if (atomicAdd(bar, 1u) == (unsigned)G - 1) {
            vb[0] = 0;
            __threadfence();
            atomicAdd(bar + 1, 1u);
        } else {
            while (vb[1] == gen) __nanosleep(20);
        }
        __threadfence();
    }
    __syncthreads();
}

__device__ __forceinline__ long long block_sum_ll(long long v, long long* red) {
    v += __shfl_xor_sync(FULL, v, 16);
    v += __shfl_xor_sync(FULL, v, 8);
    v += __shfl_xor_sync(FULL, v, 4);
    v += __shfl_xor_sync(FULL, v, 2);
    v += __shfl_xor_sync(FULL, v, 1);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    long long t = 0;
    if (threadIdx.x == 0)
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += red[w];
    return t;                            // valid in thread 0
}

// loads and stores of data other threads write: through L2 across CTAs; with one CTA the
// block barriers already order them and the L1 (write-through) serves the re-reads
template <bool ONE>
__device__ __forceinline__ int tl(const int32_t* p) { return ONE ? *p : __ldcg(p); }
template <bool ONE>
__device__ __forceinline__ void ts(int32_t* p, int v) { if (ONE) *p = v; else __stcg(p, v); }

// alive[i] != 0: local vertex i still has live edges.  oadj / iadj entries < 0 are removed.
template <bool ONE>
static __global__ void __launch_bounds__(TAIL_TH) k_tail(int32_t na, const int32_t* __restrict__ act,
                                                         const int32_t* __restrict__ optr, int32_t* oadj,
                                                         const int32_t* __restrict__ iptr, int32_t* iadj, int32_t* cin,
                                                         int32_t* cout, int32_t* kin, int32_t* kout, int32_t* alive,
                                                         int32_t* __restrict__ labels, Prio P,
                                                         const int32_t* __restrict__ orig, int first_iter, int trim,
                                                         TailTrace* T, DevCounters* dc) {
    __shared__ long long red[TAIL_TH / 32];
    const int G = gridDim.x;
    const int tid = threadIdx.x;
    // contiguous range of this thread (Gauss-Seidel along the storage order inside it)
    const int64_t nthr = (int64_t)G * blockDim.x, gt = (int64_t)blockIdx.x * blockDim.x + tid;
    const int per = (int)((na + nthr - 1) / nthr);
    const long long nl = na;
    const int lo = (int)(gt * per < nl ? gt * per : nl), hi = (int)((gt + 1) * per < nl ? (gt + 1) * per : nl);
    for (int i = lo; i < hi; i++) alive[i] = 1;
    long long live_e = 0, live_v = 0;       // block 0 thread 0: size of the current graph
    if (blockIdx.x == 0 && tid == 0) {
        live_e = optr[na];
        live_v = na;
    }
    int pass_total = 0;
    for (int iter = first_iter;; iter++) {
        // ---------------- Phase 2: passes until one changes nothing
        int pass = 0;
        for (;; pass++, pass_total++) {
            int ch = 0;
            const bool up = (pass & 1) == 0;
            for (int k = lo; k < hi; k++) {
                const int i = up ? k : hi - 1 + lo - k;
                if (!alive[i]) continue;
                const int a = tl<ONE>(cin + i), b = tl<ONE>(cout + i);
                int x = a, y = b;
                for (int e = iptr[i], ee = iptr[i + 1]; e < ee; e++) {
                    const int u = tl<ONE>(iadj + e);
                    if (u >= 0) x = max(x, tl<ONE>(cin + u));          // l.11: v_in <- max(u_in, v_in)
                }
                for (int e = optr[i], ee = optr[i + 1]; e < ee; e++) {
                    const int w = tl<ONE>(oadj + e);
                    if (w >= 0) y = max(y, tl<ONE>(cout + w));         // l.10: u_out <- max(u_out, v_out)
                }
                if (x > a) { ts<ONE>(cin + i, x); ch = 1; }
                if (y > b) { ts<ONE>(cout + i, y); ch = 1; }
            }
            if (ch) T->flag[pass_total % 3] = 1;
            if (blockIdx.x == 0 && tid == 0) {
                T->flag[(pass_total + 1) % 3] = 0;
                atomicAdd(&dc->visit_v, (unsigned long long)live_v);
                atomicAdd(&dc->visit_e, (unsigned long long)live_e);
            }
            __threadfence();
            tail_bar(T->bar, G);
            if (!*(volatile int*)&T->flag[pass_total % 3]) { pass_total++; pass++; break; }
        }
        if (blockIdx.x == 0 && tid == 0) {
            if (iter - 1 < ECL_SCC_TRACE_MAX) T->passes[iter - 1] = pass;
            T->last_iter = iter;
            long long* c = T->cnt[(iter + 2) & 3];             // the slot of iteration iter+2
            c[0] = c[1] = c[2] = 0;
        }
        long long* C = T->cnt[iter & 3];
        // ---------------- Phase 3: remove edges across different pairs or inside finished SCCs
        long long kept = 0;
        for (int i = lo; i < hi; i++) {
            if (!alive[i]) continue;
            const int a = tl<ONE>(cin + i), b = tl<ONE>(cout + i);
            const bool unfinished = a != b;
            int ko = 0, ki = 0;
            for (int e = optr[i], ee = optr[i + 1]; e < ee; e++) {
                const int w = tl<ONE>(oadj + e);
                if (w < 0) continue;
                if (unfinished && tl<ONE>(cin + w) == a && tl<ONE>(cout + w) == b) ko++;
                else ts<ONE>(oadj + e, -1);
            }
            for (int e = iptr[i], ee = iptr[i + 1]; e < ee; e++) {
                const int u = tl<ONE>(iadj + e);
                if (u < 0) continue;
                if (unfinished && tl<ONE>(cin + u) == a && tl<ONE>(cout + u) == b) ki++;
                else ts<ONE>(iadj + e, -1);
            }
            ts<ONE>(kin + i, ki);
            ts<ONE>(kout + i, ko);
            kept += ko;
        }
        kept = block_sum_ll(kept, red);
        if (tid == 0 && kept) atomicAdd((unsigned long long*)&C[0], (unsigned long long)kept);
        __threadfence();
        tail_bar(T->bar, G);
        // ---------------- Trim-1 on the kept degrees, Phase 1 reset, labels of the leavers
        long long ne = 0, nv = 0;
        for (int i = lo; i < hi; i++) {
            if (!alive[i]) continue;
            const bool tri = trim && (tl<ONE>(kin + i) == 0 || tl<ONE>(kout + i) == 0);
            int no = 0, ni = 0;
            for (int e = optr[i], ee = optr[i + 1]; e < ee; e++) {
                const int w = tl<ONE>(oadj + e);
                if (w < 0) continue;
                if (tri || (trim && (tl<ONE>(kin + w) == 0 || tl<ONE>(kout + w) == 0))) ts<ONE>(oadj + e, -1);
                else no++;
            }
            for (int e = iptr[i], ee = iptr[i + 1]; e < ee; e++) {
                const int u = tl<ONE>(iadj + e);
                if (u < 0) continue;
                if (tri || (trim && (tl<ONE>(kin + u) == 0 || tl<ONE>(kout + u) == 0))) ts<ONE>(iadj + e, -1);
                else ni++;
            }
            const int v = act ? act[i] : i;
            const int ov = orig ? orig[v] : v;
            if (no + ni > 0) {
                const int pv = (int)prio_of(P, (uint32_t)ov);
                ts<ONE>(cin + i, pv);                          // l.3-6 for the unfinished (R2)
                ts<ONE>(cout + i, pv);
                ne += no;
                nv++;
            } else {
                alive[i] = 0;
                const int a = tl<ONE>(cin + i), b = tl<ONE>(cout + i);
                labels[ov] = a == b ? (P.ids ? a : -(a + 1)) : ov;   // as k_compact_map
            }
        }
        ne = block_sum_ll(ne, red);
        nv = block_sum_ll(nv, red);
        if (tid == 0) {
            if (ne) atomicAdd((unsigned long long*)&C[1], (unsigned long long)ne);
            if (nv) atomicAdd((unsigned long long*)&C[2], (unsigned long long)nv);
        }
        __threadfence();
        tail_bar(T->bar, G);
        const long long e_next = *(volatile long long*)&C[1];
        if (blockIdx.x == 0 && tid == 0) {
            live_e = e_next;
            live_v = *(volatile long long*)&C[2];
            if (iter - 1 < ECL_SCC_TRACE_MAX) T->edges_kept[iter - 1] = *(volatile long long*)&C[0];
            if (iter < ECL_SCC_TRACE_MAX) {
                T->edges_in[iter] = live_e;
                T->vertices_in[iter] = live_v;
            }
        }
        if (e_next == 0) break;                               // no live edge: done (reading 2)
        if (iter > na + first_iter + 2) {                     // cannot happen (monotone progress)
            if (blockIdx.x == 0 && tid == 0) T->err = 1;
            break;
        }
    }
}

}  // namespace eclscc
