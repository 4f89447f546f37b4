// pack.cuh -- Phase 2 over per-iteration tile packs (k_prop_pack).
//
// The tile kernel (kernels.cuh, k_prop_tile) re-walks the CSR and CSC rows of its 2048
// vertices on every visit to find the intra-tile neighbours (16-bit slots) and the
// out-of-tile ones (global pulls); on meshes a tile is visited ~10 times per outer
// iteration and that walk -- three dependent global loads per row -- was half of the
// visit.  The working graph does not change during Phase 2, so once per outer iteration
// k_tile_pack writes each tile's shared-memory image:
//   pnin[i], pnout[i]  the slot words of local vertex i (the s_nin / s_nout encoding,
//                      SLOW_MARK for more than SLOTS intra-tile neighbours)
//   ext[off(t) ..]     the tile's cut edges as {far-end local index, v | dir << 15}:
//                      dir 0 = in-edge u -> v (v_in pulls in[u]; a raised v_out marks
//                      tile(u)), dir 1 = out-edge v -> w (v_out pulls out[w]; a raised
//                      v_in marks tile(w)); off(t) = optr[t*TT] + iptr[t*TT] (a tile
//                      never has more cut edges than edges), ext_cnt[t] entries.
// and every visit of k_prop_pack then reads its tile with coalesced vector loads and its
// cut edges as a flat list (one gather each), runs the same local fixed point
// (drain_local), and writes back / marks dirty tiles from the same list.  Alg. 1 l.10-11
// are unchanged: every live edge is either a slot pull or a cut-edge pull.
#pragma once
#include "kernels.cuh"
#include "halo.cuh"

namespace eclscc {

constexpr int PACK_TT = TILE;                 // 2048 vertices per tile
constexpr int PACK_TH = TILE_THREADS;         // 512 threads, 4 vertices each
#ifndef PACK_MINB
#define PACK_MINB 3                           // resident CTAs per SM the kernels are built for
#endif
constexpr unsigned EXT_DIR = 0x8000u;
// ECL_PROF builds: -DECL_PROF_FULL=1 (0) counts only the first (full) visits of a tile in a
// phase (only the later ones)
#ifdef ECL_PROF_FULL
#define PROF_ON(full) ((full) == ECL_PROF_FULL)
#else
#define PROF_ON(full) true
#endif
// ECL_PROF builds with -DECL_PROF_PROTO: counters 4-6 hold k_prop_async's per-visit protocol
// split instead (claims, the visit, fences + marks + finish)
#ifdef ECL_PROF_PROTO
#define PROF_PROTO 1
#else
#define PROF_PROTO 0
#endif
// Pack slot encoding: four 16-bit local indices per word; an empty slot holds PACK_TT, the
// index of a sentinel entry (value 0 <= every priority, scratch flag byte), so pulls and
// notifications run without branches; bit 63 (slot 3, only set when all four slots are
// used) marks a row with more than SLOTS intra-tile neighbours (SLOW_MARK).
constexpr unsigned long long PSLOTS_EMPTY = 0x0800080008000800ull;
static_assert(PACK_TT == 0x800, "PSLOTS_EMPTY encodes PACK_TT");
static_assert(PK_EMPTY == PSLOTS_EMPTY && PK_DIR == (int)EXT_DIR && PK_SLOW == SLOW_MARK && PACK_TT == TILE,
              "the compaction scatter writes the same pack layout (kernels.cuh PackOut)");

// tile layout in dynamic shared memory (s_in, s_out with a sentinel entry each, then the slot
// words) and the flag block (s_fin, s_fout, each with the sentinel's scratch word)
constexpr unsigned PK_OFF_OUT = (PACK_TT + 4) * 4, PK_OFF_NIN = 2 * (PACK_TT + 4) * 4,
                   PK_OFF_NOUT = PK_OFF_NIN + PACK_TT * 8, PK_OFF_FOUT = (PACK_TH + 1) * 4;
__device__ __forceinline__ unsigned smem_addr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ int ppull(const int* sig, unsigned long long src, int val) {
    const unsigned lo = (unsigned)src, hi = (unsigned)(src >> 32);
    const volatile int* s = (const volatile int*)sig;
    const int a = s[lo & 0xFFFFu], b = s[lo >> 16], c = s[hi & 0xFFFFu], d = s[(hi >> 16) & 0x7FFFu];
    return max(max(val, a), max(b, max(c, d)));
}
__device__ __forceinline__ void pnotify(unsigned long long nb, uint8_t* f) {
    const unsigned lo = (unsigned)nb, hi = (unsigned)(nb >> 32);
    volatile uint8_t* x = (volatile uint8_t*)f;
    x[lo & 0xFFFFu] = 1;
    x[lo >> 16] = 1;
    x[hi & 0xFFFFu] = 1;
    x[(hi >> 16) & 0x7FFFu] = 1;
}
// the same on 32-bit shared-window addresses (the drain's hot loop: no generic-to-shared
// conversion per access)
__device__ __forceinline__ int lds_v(unsigned a) {
    int v;
    asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long lds_v64(unsigned a) {
    unsigned long long v;
    asm volatile("ld.volatile.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void sts_v(unsigned a, int v) {
    asm volatile("st.volatile.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_b1(unsigned a) {
    asm volatile("st.volatile.shared.u8 [%0], %1;" ::"r"(a), "h"((unsigned short)1) : "memory");
}
__device__ __forceinline__ int ppull_a(unsigned sig, unsigned long long src, int val) {
    const unsigned lo = (unsigned)src, hi = (unsigned)(src >> 32);
    const int a = lds_v(sig + 4 * (lo & 0xFFFFu)), b = lds_v(sig + 4 * (lo >> 16));
    const int c = lds_v(sig + 4 * (hi & 0xFFFFu)), d = lds_v(sig + 4 * ((hi >> 16) & 0x7FFFu));
    return max(max(val, a), max(b, max(c, d)));
}
__device__ __forceinline__ void pnotify_a(unsigned long long nb, unsigned f) {
    const unsigned lo = (unsigned)nb, hi = (unsigned)(nb >> 32);
    sts_b1(f + (lo & 0xFFFFu));
    sts_b1(f + (lo >> 16));
    sts_b1(f + (hi & 0xFFFFu));
    sts_b1(f + ((hi >> 16) & 0x7FFFu));
}
// notify only the dependents a raise to `val` can change (their signature is below it): a
// dependent pulls the max of its sources, so one at or above val would pull for nothing
__device__ __forceinline__ void pnotify_sel(unsigned long long nb, unsigned f, unsigned sig, int val) {
    const unsigned lo = (unsigned)nb, hi = (unsigned)(nb >> 32);
    const unsigned s0 = lo & 0xFFFFu, s1 = lo >> 16, s2 = hi & 0xFFFFu, s3 = (hi >> 16) & 0x7FFFu;
    const int a = lds_v(sig + 4 * s0), b = lds_v(sig + 4 * s1), c = lds_v(sig + 4 * s2), d = lds_v(sig + 4 * s3);
    if (a < val) sts_b1(f + s0);
    if (b < val) sts_b1(f + s1);
    if (c < val) sts_b1(f + s2);
    if (d < val) sts_b1(f + s3);
}
// the rest of a slow row (more than SLOTS intra-tile neighbours): walk the global row
__device__ __noinline__ int pull_slow(const int* sig, const int32_t* __restrict__ ptr, const int32_t* __restrict__ adj,
                                      int base, int cnt, int v, int val) {
    for (int e = __ldg(ptr + base + v), ee = __ldg(ptr + base + v + 1); e < ee; e++) {
        const int w = __ldg(adj + e) - base;
        if ((unsigned)w < (unsigned)cnt) val = max(val, ((volatile const int*)sig)[w]);
    }
    return val;
}
__device__ __noinline__ void notify_slow(const int32_t* __restrict__ ptr, const int32_t* __restrict__ adj, int base,
                                         int cnt, int v, uint8_t* f) {
    for (int e = __ldg(ptr + base + v), ee = __ldg(ptr + base + v + 1); e < ee; e++) {
        const int w = __ldg(adj + e) - base;
        if ((unsigned)w < (unsigned)cnt) ((volatile uint8_t*)f)[w] = 1;
    }
}
__device__ __forceinline__ void pnotify_full(unsigned long long nb, const int32_t* __restrict__ ptr,
                                             const int32_t* __restrict__ adj, int base, int cnt, int v, uint8_t* f) {
    pnotify(nb, f);
    if (nb & SLOW_MARK) notify_slow(ptr, adj, base, cnt, v, f);
}

__device__ __forceinline__ unsigned gather4(unsigned w) {      // byte k (0/1) -> bit k
    return (((w & 0x01010101u) * 0x01020408u) >> 24) & 0xFu;
}

// Step 2 without the per-warp queue: in every warp round each lane pulls ONE of its flagged
// items (at most 4 vertices x 2 directions) and clears only that flag byte; its other flags
// wait for the next round.  With owner-computes pulls a round rarely holds more than one
// item per lane, so the queue's warp scan and shared-memory round trip cost more than the
// divergence they avoid (C4 Phase 2 19.5 -> 18.5 ms), and taking one item per round keeps
// every round free of a serial item loop whose length is the warp's maximum (18.5 -> 17.1 ms
// -> 15.2 ms with the packs from the scatter).  A warp leaves its rounds when none of its
// lanes has a flag left; the block rounds end when a whole block round found nothing.
// one drain item: vertex v, direction DOUT (v_out pulls from the out-neighbours and flags the
// in-neighbours; v_in the reverse), on 32-bit shared-window addresses
template <bool DOUT, bool TRICKS>
__device__ __forceinline__ void drain_item(const WGraph& g, int* __restrict__ s_sig, const int* __restrict__ s_other,
                                           const unsigned long long* __restrict__ s_src,
                                           const unsigned long long* __restrict__ s_dep, unsigned* __restrict__ s_f,
                                           unsigned a_sig, unsigned a_src, unsigned a_dep, unsigned a_f, int base,
                                           int cnt, int v, int tid, unsigned keep) {
    // clear the item's flag byte (other bytes of the word may be set concurrently): a shared
    // reduction on the 32-bit window address (atomicAnd on s_f would rebuild it from the CTA id)
    asm volatile("red.shared.and.b32 [%0], %1;" ::"r"(a_f + 4 * tid), "r"(keep) : "memory");
    const unsigned long long src = lds_v64(a_src + 8 * v);
    const int old = lds_v(a_sig + 4 * v);
    int val = ppull_a(a_sig, src, old);
    if (src & SLOW_MARK) val = pull_slow(s_sig, DOUT ? g.optr : g.iptr, DOUT ? g.oadj : g.iadj, base, cnt, v, val);
    if (val > old) {
        sts_v(a_sig + 4 * v, val);
        asm volatile("fence.acq_rel.cta;" ::: "memory");       // the value before the flags
        const unsigned long long nb = lds_v64(a_dep + 8 * v);
        pnotify_sel(nb, a_f, a_sig, val);
        if (nb & SLOW_MARK) notify_slow(DOUT ? g.iptr : g.optr, DOUT ? g.iadj : g.oadj, base, cnt, v, (uint8_t*)s_f);
        if (TRICKS && g.raise_) {
            // sound P:190: out[in[v]] (an ancestor) for v_out, in[out[v]] (a descendant) for v_in
            const int L = __ldg(g.slot + ((volatile const int*)s_other)[v]) - base;
            if ((unsigned)L < (unsigned)cnt && L != v && atomicMax(s_sig + L, val) < val) {
                __threadfence_block();
                pnotify_full(s_dep[L], DOUT ? g.iptr : g.optr, DOUT ? g.iadj : g.oadj, base, cnt, L, (uint8_t*)s_f);
            }
        }
    }
}

template <bool TRICKS = false>
__device__ __forceinline__ void drain_direct(const WGraph& g, int* __restrict__ s_in, int* __restrict__ s_out,
                                             const unsigned long long* __restrict__ s_nin,
                                             const unsigned long long* __restrict__ s_nout,
                                             unsigned* __restrict__ s_fin, unsigned* __restrict__ s_fout, int base,
                                             int cnt, unsigned& prof_rounds, unsigned& prof_drains,
                                             unsigned& prof_pushes) {
    const int tid = threadIdx.x;
    const int v0 = tid * VPT;
    // two base registers (the tile layout and the flag words are each one block; see the
    // kernels): every other address is a constant offset, so the loop does not rebuild
    // shared-window addresses per access
    // (through a shuffle: ptxas would otherwise re-derive them from the CTA id before each use)
    const unsigned a_in = __shfl_sync(FULL, smem_addr(s_in), 0), a_fin = __shfl_sync(FULL, smem_addr(s_fin), 0);
    const unsigned a_out = a_in + PK_OFF_OUT, a_nin = a_in + PK_OFF_NIN, a_nout = a_in + PK_OFF_NOUT;
    const unsigned a_fout = a_fin + PK_OFF_FOUT;
    for (;;) {
        int worked = 0;
#ifdef ECL_PROF
        if (tid == 0) prof_rounds++;
#endif
        for (;;) {
#ifdef ECL_PROF
            if ((tid & 31) == 0) prof_drains++;
#endif
            const unsigned ii = gather4((unsigned)lds_v(a_fin + 4 * tid));
            const unsigned oo = gather4((unsigned)lds_v(a_fout + 4 * tid));
            if (!__any_sync(FULL, (ii | oo) != 0)) break;
            // one v_in item AND one v_out item per lane and round: a warp holding both kinds
            // runs both paths anyway (divergence), so a lane with both does both
            if (ii | oo) {
                worked = 1;
#ifdef ECL_PROF
                prof_pushes += (ii != 0) + (oo != 0);
#endif
            }
            if (ii) {
                const int k = __ffs(ii) - 1;
                drain_item<false, TRICKS>(g, s_in, s_out, s_nin, s_nout, s_fin, a_in, a_nin, a_nout, a_fin, base, cnt,
                                          v0 + k, tid, ~(0xFFu << (8 * k)));
            }
            if (oo) {
                const int k = __ffs(oo) - 1;
                drain_item<true, TRICKS>(g, s_out, s_in, s_nout, s_nin, s_fout, a_out, a_nout, a_nin, a_fout, base, cnt,
                                         v0 + k, tid, ~(0xFFu << (8 * k)));
            }
            __syncwarp();
        }
        if (!__syncthreads_or(worked)) break;
    }
}

constexpr size_t pack_dyn_smem() { return (size_t)(PACK_TT + 4) * 4 * 2 + (size_t)PACK_TT * 8 * 2; }

// one CTA per tile: slot words and cut-edge list (graphs without rows longer than HEAVY_T)
static __global__ void __launch_bounds__(PACK_TH) k_tile_pack(WGraph g, unsigned long long* __restrict__ pnin,
                                                              unsigned long long* __restrict__ pnout,
                                                              int2* __restrict__ ext, int* __restrict__ ext_cnt) {
    __shared__ int s_n;
    const int tid = threadIdx.x, tile = blockIdx.x;
    const int base = tile * PACK_TT, cnt = min(PACK_TT, g.na - base);
    const int64_t off = (int64_t)__ldg(g.optr + base) + __ldg(g.iptr + base);
    if (tid == 0) s_n = 0;
    __syncthreads();
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int v = tid * VPT + k;
        unsigned long long ni = PSLOTS_EMPTY, no = PSLOTS_EMPTY;
        if (v < cnt) {
            const int gi = base + v;
            int ns = 0;
            for (int e = __ldg(g.iptr + gi), ee = __ldg(g.iptr + gi + 1); e < ee; e++) {
                const int u = __ldg(g.iadj + e);
                if ((unsigned)(u - base) >= (unsigned)cnt) {
                    ext[off + atomicAdd(&s_n, 1)] = make_int2(u, v);
                    continue;
                }
                if (ns < SLOTS) add_slot(ni, ns, (unsigned)(u - base));
                else ni |= SLOW_MARK;
            }
            ns = 0;
            for (int e = __ldg(g.optr + gi), ee = __ldg(g.optr + gi + 1); e < ee; e++) {
                const int w = __ldg(g.oadj + e);
                if ((unsigned)(w - base) >= (unsigned)cnt) {
                    ext[off + atomicAdd(&s_n, 1)] = make_int2(w, v | (int)EXT_DIR);
                    continue;
                }
                if (ns < SLOTS) add_slot(no, ns, (unsigned)(w - base));
                else no |= SLOW_MARK;
            }
        }
        pnin[(int64_t)base + v] = ni;       // the pack arrays are padded to whole tiles
        pnout[(int64_t)base + v] = no;
    }
    __syncthreads();
    if (tid == 0) ext_cnt[tile] = s_n;
}

// ---- bulk (TMA) copies of a tile's pack rows into shared memory (cp.async.bulk, SASS
// UBLKCP) completing on an mbarrier.  The pack is read-only during Phase 2, so the slot
// words of the NEXT tile of a CTA's run are copied while the current one writes back and
// marks (its drain no longer reads them); the visit waits on the barrier only after its
// own value loads and cut-edge pulls.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
    asm volatile(
        "{\n .reg .pred p;\n"
        "WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
// one thread: the pack rows of `tile` -> s_nin / s_nout (2 x 16 KB), completion on bar
__device__ __forceinline__ void pack_issue(const unsigned long long* __restrict__ pnin,
                                           const unsigned long long* __restrict__ pnout, int tile,
                                           unsigned long long* s_nin, unsigned long long* s_nout,
                                           unsigned long long* bar) {
    constexpr unsigned BYTES = PACK_TT * 8;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // earlier generic reads first
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(2 * BYTES)
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(s_nin)),
                 "l"(pnin + (int64_t)tile * PACK_TT), "r"(BYTES), "r"(smem_u32(bar))
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(s_nout)),
                 "l"(pnout + (int64_t)tile * PACK_TT), "r"(BYTES), "r"(smem_u32(bar))
                 : "memory");
}
// the bulk-copy state of a CTA: its barrier, the parity of the next phase, and whether the
// current tile's copy was already issued by the previous visit
struct PackTma {
    unsigned long long* bar;
    unsigned phase;
    bool issued;
};

// One visit of tile `tile` from its pack.  Returns non-zero in every thread if a
// signature was raised.  T (k_prop_async): the pack rows arrive by bulk copy (PackTma);
// otherwise (k_prop_pack) by vector loads.
template <typename Mark, bool HALO = false, bool TRICKS = false>
__device__ __forceinline__ int pack_visit(const WGraph& g, int32_t* __restrict__ cin, int32_t* __restrict__ cout,
                                          const unsigned long long* __restrict__ pnin,
                                          const unsigned long long* __restrict__ pnout, const int2* __restrict__ ext,
                                          const int* __restrict__ ext_cnt, DevCounters* __restrict__ dc, int tile,
                                          int full, Mark mark, const TileSmem<PACK_TT>& S, int next = -1,
                                          PackTma* T = nullptr, const HaloPush* H = nullptr) {
    int* s_in = S.s_in;
    int* s_out = S.s_out;
    unsigned long long* s_nin = S.s_nin;
    unsigned long long* s_nout = S.s_nout;
    unsigned* s_fin = S.s_fin;
    unsigned* s_fout = S.s_fout;
    const int tid = threadIdx.x;
    const int base = tile * PACK_TT;
    const int cnt = min(PACK_TT, g.na - base);
    const int v0 = tid * VPT;
    const int ne = __ldg(ext_cnt + tile);
    const int2* E = ext + (int64_t)__ldg(g.optr + base) + __ldg(g.iptr + base);
#ifdef ECL_PROF
    const long long t_start = clock64();
    if (tid == 0 && PROF_ON(full)) PROF_ADD(dc, 0, 1);
#endif

    // ---- step 1: own values and slot words (coalesced 16-byte loads, or the bulk copy),
    // then the cut-edge pulls (Alg. 1 l.10-11 across the tile boundary), folded in with
    // shared atomicMax
    if (T) {
        if (!T->issued && tid == 0) pack_issue(pnin, pnout, tile, s_nin, s_nout, T->bar);
    } else {
        const ulonglong2* a = (const ulonglong2*)(pnin + base + v0);
        const ulonglong2* b = (const ulonglong2*)(pnout + base + v0);
        ulonglong2* sa = (ulonglong2*)(s_nin + v0);
        ulonglong2* sb = (ulonglong2*)(s_nout + v0);
        sa[0] = __ldg(a);
        sa[1] = __ldg(a + 1);
        sb[0] = __ldg(b);
        sb[1] = __ldg(b + 1);
    }
    int x0[VPT], y0[VPT];
    {
        if (v0 + VPT <= cnt) {
            const int4 x = __ldcg((const int4*)(cin + base + v0));
            const int4 y = __ldcg((const int4*)(cout + base + v0));
            x0[0] = x.x; x0[1] = x.y; x0[2] = x.z; x0[3] = x.w;
            y0[0] = y.x; y0[1] = y.y; y0[2] = y.z; y0[3] = y.w;
        } else {
#pragma unroll
            for (int k = 0; k < VPT; k++) {
                x0[k] = v0 + k < cnt ? ld_cg(cin + base + v0 + k) : 0;
                y0[k] = v0 + k < cnt ? ld_cg(cout + base + v0 + k) : 0;
            }
        }
        *(int4*)(s_in + v0) = make_int4(x0[0], x0[1], x0[2], x0[3]);
        *(int4*)(s_out + v0) = make_int4(y0[0], y0[1], y0[2], y0[3]);
    }
    if (tid == 0) {                                   // roofline accounting (SURVEY 8(d) terms)
        S.s_acc[0] += (unsigned long long)cnt;        // per CTA; the kernel adds it to dc once
        S.s_acc[1] += (unsigned long long)(__ldg(g.optr + base + cnt) - __ldg(g.optr + base));
    }
    __syncthreads();
    for (int i = tid; i < ne; i += PACK_TH) {
        const int2 e = __ldg(E + i);
        const int v = e.y & 0x7FFF;
        int* sig = (e.y & EXT_DIR) ? s_out : s_in;
        const int32_t* gsig = (e.y & EXT_DIR) ? cout : cin;
        int val = ld_cg(gsig + e.x);
        // path compression: in[in[u]] / out[out[w]] -- the signature of the vertex whose
        // priority u carries, an ancestor (descendant) of u, so never worse than in[u]
        if (TRICKS && g.compress) val = max(val, ld_cg(gsig + __ldg(g.slot + val)));
        if (val > ((volatile int*)sig)[v]) atomicMax(sig + v, val);
    }
    __syncthreads();
    if (T) {                                          // the slot words have landed
        mbar_wait(T->bar, T->phase);
        T->phase ^= 1u;
    }
    // ---- step 1b: flags.  First visit of a phase: every vertex; otherwise the intra-tile
    // dependents of what the cut-edge pulls raised.
    unsigned fin = 0, fout = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        if (v0 + k >= cnt) continue;
        if (full || s_in[v0 + k] > x0[k]) fin |= 1u << (8 * k);
        if (full || s_out[v0 + k] > y0[k]) fout |= 1u << (8 * k);
    }
    s_fin[tid] = full ? fin : 0u;
    s_fout[tid] = full ? fout : 0u;
    __syncthreads();
    if (!full && (fin | fout)) {
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            const int v = v0 + k;
            if ((fin >> (8 * k)) & 0xFF) pnotify_full(s_nout[v], g.optr, g.oadj, base, cnt, v, (uint8_t*)s_fin);
            if ((fout >> (8 * k)) & 0xFF) pnotify_full(s_nin[v], g.iptr, g.iadj, base, cnt, v, (uint8_t*)s_fout);
        }
    }
    __syncthreads();
    // the next tile of this CTA's run: pull its pack rows and values into L2 while this one
    // drains (384 lines of 128 B, one per thread; L2 is coherent, so racing writers are fine)
    if (next >= 0 && tid < 384 && (!T || tid >= 256)) {   // (with T the pack arrives by bulk copy)
        const int nb = next * PACK_TT;
        const char* line;
        if (tid < 128) line = (const char*)(pnin + nb) + 128 * tid;
        else if (tid < 256) line = (const char*)(pnout + nb) + 128 * (tid - 128);
        else if (tid < 320) line = (const char*)(cin + nb) + 128 * (tid - 256);
        else line = (const char*)(cout + nb) + 128 * (tid - 320);
        if (tid < 256 || nb + 32 * ((tid - 256) & 63) < g.na)
            asm volatile("prefetch.global.L2 [%0];" ::"l"(line));
    }
    // ---- step 2: local fixed point in shared memory (same drain loop as k_prop_tile)
#ifdef ECL_PROF
    const long long t_step1 = clock64();
#endif
    {
        unsigned r0 = 0, r1 = 0, r2 = 0;
        drain_direct<TRICKS>(g, s_in, s_out, s_nin, s_nout, s_fin, s_fout, base, cnt, r0, r1, r2);
#ifdef ECL_PROF
        r2 = warp_sum(r2);
        if ((tid & 31) == 0 && PROF_ON(full)) { PROF_ADD(dc, 2, r1); PROF_ADD(dc, 3, r2); }
        if (tid == 0 && PROF_ON(full)) PROF_ADD(dc, 1, r0);
#endif
    }
#ifdef ECL_PROF
    __syncthreads();
    const long long t_step2 = clock64();
#endif
    // the drain is over (its last block barrier passed): the slot words are free, so the next
    // tile's copy overlaps this write-back and the marks
    if (T) {
        T->issued = next >= 0;
        if (next >= 0 && tid == 0) pack_issue(pnin, pnout, next, s_nin, s_nout, T->bar);
    }
    // ---- step 3: write back (whole 16-byte groups; only this CTA writes these vertices
    // during the pass, so global memory still holds the originals: re-read rather than
    // kept in registers across step 2) and record which directions rose, for the marks
    unsigned rin = 0, rout = 0;
    if (v0 + VPT <= cnt) {
        const int4 xs = *(const int4*)(s_in + v0);
        const int4 a = __ldcg((const int4*)(cin + base + v0));
        rin = (xs.x > a.x ? 1u : 0u) | (xs.y > a.y ? 0x100u : 0u) | (xs.z > a.z ? 0x10000u : 0u) |
              (xs.w > a.w ? 0x1000000u : 0u);
        if (rin) __stcg((int4*)(cin + base + v0), xs);
        const int4 ys = *(const int4*)(s_out + v0);
        const int4 b = __ldcg((const int4*)(cout + base + v0));
        rout = (ys.x > b.x ? 1u : 0u) | (ys.y > b.y ? 0x100u : 0u) | (ys.z > b.z ? 0x10000u : 0u) |
               (ys.w > b.w ? 0x1000000u : 0u);
        if (rout) __stcg((int4*)(cout + base + v0), ys);
    } else {
        for (int k = 0; k < VPT && v0 + k < cnt; k++) {
            const int gi = base + v0 + k;
            const int xv = s_in[v0 + k], yv = s_out[v0 + k];
            if (xv > ld_cg(cin + gi)) { cin[gi] = xv; rin |= 1u << (8 * k); }
            if (yv > ld_cg(cout + gi)) { cout[gi] = yv; rout |= 1u << (8 * k); }
        }
    }
    // partitioned mode (halo.cuh, f1): every raised halo copy goes straight into every rank's
    // exchange buffer (remote atomic max / multimem reduction), overlapping this rank's
    // fixed point tile by tile
    if (HALO && (rin | rout)) {
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            const unsigned bi = (rin >> (8 * k)) & 1u, bo = (rout >> (8 * k)) & 1u;
            if (!(bi | bo)) continue;
            const int p = __ldg(H->hpos + base + v0 + k);
            if (p < 0) continue;
            if (bi) halo_push_one(*H, 2 * (int64_t)p, s_in[v0 + k]);
            if (bo) halo_push_one(*H, 2 * (int64_t)p + 1, s_out[v0 + k]);
        }
    }
    const int any = __syncthreads_or((int)(rin | rout));   // also: every drain flag is consumed
#ifdef ECL_PROF
    {
        const int nr = warp_sum(__popc(rin) + __popc(rout));   // raised vertex-directions
        if ((tid & 31) == 0 && nr && PROF_ON(full)) PROF_ADD(dc, 7, nr);
    }
#endif
    if (any && mark.on()) {
        s_fin[tid] = rin;
        s_fout[tid] = rout;
        __syncthreads();
        const uint8_t* bi = (const uint8_t*)s_fin;
        const uint8_t* bo = (const uint8_t*)s_fout;
        for (int i = tid; i < ne; i += PACK_TH) {
            const int2 e = __ldg(E + i);
            const int v = e.y & 0x7FFF;
            // in-edge u -> v: a raised v_out reaches u; out-edge v -> w: a raised v_in reaches w
            if (((e.y & EXT_DIR) ? bi[v] : bo[v]) != 0) mark(e.x / PACK_TT);
        }
    }
#ifdef ECL_PROF
    __syncthreads();
    if (tid == 0 && PROF_ON(full) && !PROF_PROTO) {
        const long long t_end = clock64();
        PROF_ADD(dc, 4, t_step1 - t_start);
        PROF_ADD(dc, 5, t_step2 - t_step1);
        PROF_ADD(dc, 6, t_end - t_step2);
    }
#endif
    return any;
}

// Phase-2 pass over the packs (pass protocol, dirty skipping and runs as k_prop_tile)
template <bool TRICKS>
static __global__ void __launch_bounds__(PACK_TH, PACK_MINB)
k_prop_pack(WGraph g, int32_t* __restrict__ cin, int32_t* __restrict__ cout, const unsigned long long* __restrict__ pnin,
            const unsigned long long* __restrict__ pnout, const int2* __restrict__ ext, const int* __restrict__ ext_cnt,
            DevCounters* __restrict__ dc, int pass, int first, uint8_t* __restrict__ dirty_cur,
            uint8_t* __restrict__ dirty_next, int full, int run) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ unsigned s_flags[2 * (PACK_TH + 1)];                   // s_fin, s_fout (+ the sentinel's scratch byte)
    unsigned* s_fin = s_flags;
    unsigned* s_fout = s_flags + PACK_TH + 1;
    __shared__ int s_dirty;
    TileSmem<PACK_TT> S;
    S.s_in = (int*)smem_raw;                                          // [PACK_TT] + sentinel
    S.s_out = S.s_in + PACK_TT + 4;
    S.s_nin = (unsigned long long*)(S.s_out + PACK_TT + 4);
    S.s_nout = S.s_nin + PACK_TT;
    __shared__ unsigned long long s_acc[3];
    if (threadIdx.x == 0) { S.s_in[PACK_TT] = 0; S.s_out[PACK_TT] = 0; s_acc[0] = s_acc[1] = s_acc[2] = 0; }
    S.s_fin = s_fin;
    S.s_fout = s_fout;
    S.s_queue = nullptr;
    S.s_acc = s_acc;
    if (!pass_begin(dc, pass, first)) return;
    const int ntiles = (g.na + PACK_TT - 1) / PACK_TT;
    const int tid = threadIdx.x;
    int ch_any = 0;
    for (int j = 0; j < run; j++) {
        const int idx = (int)blockIdx.x * run + ((pass & 1) ? run - 1 - j : j);
        if (idx >= ntiles) continue;
        const int tile = (pass & 1) ? ntiles - 1 - idx : idx;
        if (dirty_cur) {
            if (tid == 0) {
                s_dirty = dirty_cur[tile];
                dirty_cur[tile] = 0;
            }
            __syncthreads();
            const int d = s_dirty;
            __syncthreads();
            if (!d) continue;
        }
        ch_any |= pack_visit<MarkNext, false, TRICKS>(g, cin, cout, pnin, pnout, ext, ext_cnt, dc, tile, full,
                                                      MarkNext{dirty_next}, S);
        __syncthreads();
    }
    if (ch_any && tid == 0) dc->changed[pass & (RING - 1)] = 1;
    if (tid == 0 && s_acc[0]) {
        atomicAdd(&dc->visit_v, s_acc[0]);
        atomicAdd(&dc->visit_e, s_acc[1]);
    }
}

// ------------------------------------------------------------------ asynchronous mode
// Phase 2 as ONE persistent launch per outer iteration ("asynchronous", P:204
// "persistent threads") at tile granularity, without pass barriers.  A global sweep cursor
// runs over the tiles, ascending and descending in turn (the alternating pass order of
// k_prop_pack); resident CTAs claim the next dirty tile under the cursor, so a tile
// dirtied ahead of the cursor is visited in the same sweep (Gauss-Seidel between tiles)
// and no CTA waits for the slowest visit of a pass.
// Tile state machine (tstate): 0 clean, 1 dirty, 2 running, 3 running + dirtied again.
//   mark(t):   0 -> 1 or 2 -> 3 (pending++ either way); 1, 3 unchanged
//   claim(t):  1 -> 2 (the first visit of a tile in the phase is a full one)
//   finish(t): 2 -> 0; 3 -> 1 (state -= 2)
// pending = #state 1 + #state 2 + 2 * #state 3, so every state change by a mark (0 -> 1,
// 2 -> 3) adds one and every finish subtracts one: the finish is two fire-and-forget
// reductions (no compare-and-swap round trip in the visit loop), and pending == 0 still
// means no tile is dirty or running.  A visit's marks (pending++) precede its own finish
// (pending--), so pending == 0 means no visit is running and every tile's last visit saw
// its final inputs: the Phase-2 fixed point (Alg. 1 l.7-14).  Values are
// written (st.cg) and fenced before the marks; a claimer fences after its claim and reads
// through L2, so it sees every value written before the state change it observed.
// the cursor, the pending count and the stop word sit in separate 128-byte lines: claimers
// hammer the cursor while visits count marks and finishes on the pending word
constexpr int AQ_CUR = 0, AQ_PEND = 16, AQ_STOP = 32, AQ_WORDS = 48;
struct AsyncQ {
    int* tstate;                  // [ntiles]
    uint8_t* tseen;               // [ntiles] visited in this phase
    unsigned long long* ctr;      // [AQ_CUR] cursor, [AQ_PEND] pending, [AQ_STOP] stop
};
__device__ __forceinline__ void aq_mark(const AsyncQ& Q, int t) {
    int st = 0;                                   // (try clean first: no separate read)
    for (;;) {
        const int old = atomicCAS(Q.tstate + t, st, st == 0 ? 1 : 3);
        if (old == st) break;
        if (old == 1 || old == 3) return;         // already dirty
        st = old;
    }
    atomicAdd(Q.ctr + AQ_PEND, 1ull);             // 0 -> 1 or 2 -> 3
}
// the end of a visit (after its marks): 2 -> 0 or 3 -> 1, pending - 1
__device__ __forceinline__ void aq_finish(const AsyncQ& Q, int t) {
    atomicSub(Q.tstate + t, 2);
    atomicAdd(Q.ctr + AQ_PEND, ~0ull);
}
static __global__ void k_async_init(AsyncQ Q, int ntiles) {
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < ntiles; t += gridDim.x * blockDim.x) {
        Q.tstate[t] = 1;
        Q.tseen[t] = 0;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) { Q.ctr[AQ_CUR] = 0; Q.ctr[AQ_PEND] = (unsigned long long)ntiles; Q.ctr[AQ_STOP] = 0; }
}

constexpr int CLAIM_MAX = 32;     // sweep positions per claim (a CTA's run of tiles), <= a warp

// marks of one visit, deduplicated per neighbour tile in a shared-memory hash set
constexpr int MSET = 256;
struct MarkSet {
    int* set;
    AsyncQ Q;
    __device__ __forceinline__ bool on() const { return true; }
    __device__ __forceinline__ void operator()(int t) const {
        unsigned h = ((unsigned)t * 0x9E3779B1u) >> 24;          // MSET = 256 slots
        for (int k = 0; k < 16; k++, h = (h + 1) & (MSET - 1)) {
            const int cur = ((volatile int*)set)[h];
            if (cur == t) return;
            if (cur == -1) {
                const int old = atomicCAS(set + h, -1, t);
                if (old == -1 || old == t) return;
            }
        }
        __threadfence();                                          // crowded set: mark directly
        aq_mark(Q, t);
    }
};

// warp 0 of a CTA (all 32 lanes): one cursor step covers `claim` consecutive sweep positions;
// every dirty tile among them is claimed (1 -> 2) into s_claim / s_seen in sweep order.
// Returns the number claimed (0: the fixed point, or the stop word).
__device__ __forceinline__ int aq_claim(const AsyncQ& Q, int ntiles, int claim, int lane, int* s_claim,
                                        uint8_t* s_seen, long long& t0, DevCounters* dc) {
    int got = 0, stop = 0;
    volatile unsigned long long* ctr = Q.ctr;
    for (unsigned miss = 0;; miss += claim) {
        // the stop words and the cursor step are requested together (one round trip);
        // positions taken after the fixed point are harmless
        unsigned long long pos = 0;
        if (lane == 0) {
            const unsigned long long pend = ctr[AQ_PEND], halt = ctr[AQ_STOP];
            pos = atomicAdd(Q.ctr + AQ_CUR, (unsigned long long)claim);
            stop = (pend == 0 || halt) ? 1 : 0;           // fixed point / watchdog
        }
        if (__shfl_sync(FULL, stop, 0)) break;
        pos = __shfl_sync(FULL, pos, 0) + (unsigned)lane;
        bool mine = false;
        int c = 0, seen = 0;
        if (lane < claim) {
            const unsigned long long k = pos / (unsigned)ntiles;
            const int off = (int)(pos - k * (unsigned)ntiles);
            c = (k & 1) ? ntiles - 1 - off : off;
            // the seen byte is read with the claim (a tile visited between this read and
            // the claim only gets one extra full visit); the claim is the compare-and-swap
            // itself, with no separate read of the state first (one L2 round trip less)
            seen = ((volatile uint8_t*)Q.tseen)[c];
            mine = atomicCAS(Q.tstate + c, 1, 2) == 1;
        }
        const unsigned m = __ballot_sync(FULL, mine);
        if (mine) {
            const int slot = __popc(m & ((1u << lane) - 1));
            s_claim[slot] = c;

            s_seen[slot] = (uint8_t)seen;
            if (!seen) Q.tseen[c] = 1;
        }
        if (m) { got = __popc(m); break; }
        if (miss >= (unsigned)ntiles) {                    // a whole sweep without work
            __nanosleep(256);
            if (lane == 0 && clock64() - t0 > (1ll << 36)) {   // ~30 s idle: protocol bug
                atomicExch(&dc->err, 3);
                atomicExch(Q.ctr + AQ_STOP, 1ull);
            }
        }
    }
    return got;
}

template <bool HALO, bool TRICKS>
static __global__ void __launch_bounds__(PACK_TH, PACK_MINB)
k_prop_async(WGraph g, int32_t* __restrict__ cin, int32_t* __restrict__ cout, const unsigned long long* __restrict__ pnin,
             const unsigned long long* __restrict__ pnout, const int2* __restrict__ ext, const int* __restrict__ ext_cnt,
             DevCounters* __restrict__ dc, AsyncQ Q, int claim, const __grid_constant__ HaloPush H) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ unsigned s_flags[2 * (PACK_TH + 1)];                   // s_fin, s_fout (drain_direct layout)
    unsigned* s_fin = s_flags;
    unsigned* s_fout = s_flags + PACK_TH + 1;
    __shared__ int s_set[MSET];
    __shared__ int s_claim[CLAIM_MAX], s_nclaim;
    __shared__ uint8_t s_seen[CLAIM_MAX];
    TileSmem<PACK_TT> S;
    S.s_in = (int*)smem_raw;
    S.s_out = S.s_in + PACK_TT + 4;
    S.s_nin = (unsigned long long*)(S.s_out + PACK_TT + 4);
    S.s_nout = S.s_nin + PACK_TT;
    __shared__ unsigned long long s_acc[3];            // visited vertices, edges, tiles (flushed at the end)
    __shared__ __align__(8) unsigned long long s_bar;  // bulk-copy barrier of the pack rows
    S.s_fin = s_fin;
    S.s_fout = s_fout;
    S.s_queue = nullptr;
    S.s_acc = s_acc;
    const int tid = threadIdx.x;
    const int ntiles = (g.na + PACK_TT - 1) / PACK_TT;
    if (tid == 0) {
        S.s_in[PACK_TT] = 0; S.s_out[PACK_TT] = 0; s_acc[0] = s_acc[1] = s_acc[2] = 0;
        mbar_init(&s_bar, 1);
    }
    PackTma T{&s_bar, 0u, false};
    long long t0 = clock64();
    for (;;) {
        // warp 0 claims: one cursor step covers CLAIM consecutive sweep positions, every
        // dirty tile among them is claimed and the CTA visits them in sweep order (a run)
#ifdef ECL_PROF
        const long long t_claim = clock64();
#endif
        if (tid < 32) {
            const int lane = tid;
            const int got = aq_claim(Q, ntiles, claim, lane, s_claim, s_seen, t0, dc);
            if (lane == 0) {
                s_nclaim = got;
                s_acc[2] += (unsigned long long)got;       // tile visits of the phase
                if (got) t0 = clock64();
            }
            __threadfence();                                      // claims before the value reads
        }
        __syncthreads();
#ifdef ECL_PROF
        long long tp = clock64();
        if (tid == 0 && PROF_PROTO) PROF_ADD(dc, 4, tp - t_claim);
#endif
        const int nclaim = s_nclaim;
        if (nclaim == 0) break;
        for (int j = 0; j < nclaim; j++) {
            const int tile = s_claim[j], full = s_seen[j] == 0;
            for (int i = tid; i < MSET; i += PACK_TH) s_set[i] = -1;
            __syncthreads();
            pack_visit<MarkSet, HALO, TRICKS>(g, cin, cout, pnin, pnout, ext, ext_cnt, dc, tile, full, MarkSet{s_set, Q}, S,
                                      j + 1 < nclaim ? s_claim[j + 1] : -1, &T, HALO ? &H : nullptr);
#ifdef ECL_PROF
            const long long tv = clock64();
            if (tid == 0 && PROF_PROTO) PROF_ADD(dc, 5, tv - tp);
#endif
            __threadfence();                                      // values before marks
            __syncthreads();
            for (int i = tid; i < MSET; i += PACK_TH)
                if (s_set[i] >= 0) aq_mark(Q, s_set[i]);
            __threadfence();
            __syncthreads();                                      // marks (pending++) before finish
            if (tid == 0) {
                aq_finish(Q, tile);
            }
#ifdef ECL_PROF
            tp = clock64();
            if (tid == 0 && PROF_PROTO) PROF_ADD(dc, 6, tp - tv);
#endif
        }
        __syncthreads();                                          // s_claim is rewritten next
    }
    if (tid == 0) {
        if (s_acc[0]) atomicAdd(&dc->visit_v, s_acc[0]);
        if (s_acc[1]) atomicAdd(&dc->visit_e, s_acc[1]);
        if (s_acc[2]) atomicAdd(&dc->passes, s_acc[2]);
    }
    if (HALO && H.sys) __threadfence_system();          // pushes to other GPUs before the barrier
}

}  // namespace eclscc
