// cluster.cuh -- Phase 2 with thread-block-cluster tiles (ECL_SCC_CLUSTER).
//
// A CTA pair (cluster of 2, `__cluster_dims__(2,1,1)`) runs the block-local fixed point of
// one PAIR TILE of 4096 consecutive local vertices: CTA rank r holds half r (2048 vertices,
// the same shared-memory image as a k_prop_async tile) and reaches the other half through
// distributed shared memory (DSMEM, generic pointers from `mapa`).  Edges between the two
// halves are therefore intra-tile: they propagate inside one visit instead of through a
// global re-visit (P:192 block-local iteration over a larger block).
//
// Pack of a pair tile (k_pack_pair): slot words as in pack.cuh but RELATIVE TO THE HALF of
// the row's vertex: a slot is the neighbour's index inside its half, with bit 12 (PAIR_REMOTE)
// set when the neighbour is in the other half; an empty slot is the own half's sentinel
// (index 2048).  Cut edges (leaving the pair tile) form one flat list per pair tile,
// {far-end local index, v | dir << 15} with v pair-local.
//
// Visit (k_prop_cluster):
//   1. each CTA bulk-copies its half's pack rows, loads its half's values and pulls the cut
//      edges of its own vertices; cluster barrier (both halves' values are in place);
//   2. drain: as pack.cuh's drain_direct, a flagged vertex pulls its slots -- local ones from
//      its CTA's shared memory, remote ones through DSMEM -- and on a raise flags its
//      dependents in either half (remote flags by DSMEM byte stores, ordered after the value by
//      a cluster-scope fence).  Rounds end with a cluster barrier that ORs "worked" over both
//      CTAs (a flag set in a finished partner is seen in the next round);
//   3. each CTA writes back its half and marks the pair tiles of its raised cut-edge ends.
// Claims, tile states and the pending count are those of pack.cuh (AsyncQ) over pair tiles;
// rank 0 claims and hands the run to rank 1 through DSMEM.
#pragma once
#include <cooperative_groups.h>

#include "pack.cuh"

namespace eclscc {

namespace cg = cooperative_groups;

constexpr int PAIR_TT = 2 * PACK_TT;          // vertices per pair tile
constexpr unsigned PAIR_REMOTE = 0x1000u;     // slot bit: the neighbour is in the other half
constexpr unsigned long long PAIR_EMPTY = 0x0800080008000800ull;   // four own-half sentinels

__device__ __forceinline__ void fence_cluster() { asm volatile("fence.acq_rel.cluster;" ::: "memory"); }

// pack rows of pair tiles (one CTA of PACK_TH threads per pair tile, 8 vertices per thread)
static __global__ void __launch_bounds__(PACK_TH) k_pack_pair(WGraph g, unsigned long long* __restrict__ pnin,
                                                              unsigned long long* __restrict__ pnout,
                                                              int2* __restrict__ ext, int* __restrict__ ext_cnt) {
    __shared__ int s_n;
    const int tid = threadIdx.x, tile = blockIdx.x;
    const int base = tile * PAIR_TT, cnt = min(PAIR_TT, g.na - base);
    const int64_t off = (int64_t)__ldg(g.optr + base) + __ldg(g.iptr + base);
    if (tid == 0) s_n = 0;
    __syncthreads();
    for (int k = 0; k < PAIR_TT / PACK_TH; k++) {
        const int v = k * PACK_TH + tid;
        unsigned long long ni = PAIR_EMPTY, no = PAIR_EMPTY;
        if (v < cnt) {
            const int gi = base + v, half = v / PACK_TT;
            int ns = 0;
            for (int e = __ldg(g.iptr + gi), ee = __ldg(g.iptr + gi + 1); e < ee; e++) {
                const int u = __ldg(g.iadj + e) - base;
                if ((unsigned)u >= (unsigned)cnt) {
                    ext[off + atomicAdd(&s_n, 1)] = make_int2(u + base, v);
                    continue;
                }
                const unsigned sl = (unsigned)(u % PACK_TT) | (u / PACK_TT != half ? PAIR_REMOTE : 0u);
                if (ns < SLOTS) add_slot(ni, ns, sl);
                else ni |= SLOW_MARK;
            }
            ns = 0;
            for (int e = __ldg(g.optr + gi), ee = __ldg(g.optr + gi + 1); e < ee; e++) {
                const int w = __ldg(g.oadj + e) - base;
                if ((unsigned)w >= (unsigned)cnt) {
                    ext[off + atomicAdd(&s_n, 1)] = make_int2(w + base, v | (int)EXT_DIR);
                    continue;
                }
                const unsigned sl = (unsigned)(w % PACK_TT) | (w / PACK_TT != half ? PAIR_REMOTE : 0u);
                if (ns < SLOTS) add_slot(no, ns, sl);
                else no |= SLOW_MARK;
            }
        }
        pnin[(int64_t)base + v] = ni;       // the pack arrays cover whole pair tiles
        pnout[(int64_t)base + v] = no;
    }
    __syncthreads();
    if (tid == 0) ext_cnt[tile] = s_n;
}

// a slot of a half-relative slot word: (own or partner) array + index
__device__ __forceinline__ int pair_ld(const int* own, const int* rem, unsigned s) {
    const int* b = (s & PAIR_REMOTE) ? rem : own;
    return ((const volatile int*)b)[s & 0xFFFu];
}
__device__ __forceinline__ int pair_pull(const int* own, const int* rem, unsigned long long src, int val) {
    const unsigned lo = (unsigned)src, hi = (unsigned)(src >> 32);
    const int a = pair_ld(own, rem, lo & 0xFFFFu), b = pair_ld(own, rem, lo >> 16),
              c = pair_ld(own, rem, hi & 0xFFFFu), d = pair_ld(own, rem, (hi >> 16) & 0x7FFFu);
    return max(max(val, a), max(b, max(c, d)));
}
// a flag in the partner's shared memory is set with a DSMEM atomic on its flag word: a plain
// remote byte store is not atomic with the owner's atomicAnd on the same word (measured: lost
// notifications)
__device__ __forceinline__ void pair_set(uint8_t* own, uint8_t* rem, unsigned s) {
    const unsigned i = s & 0xFFFu;
    if (s & PAIR_REMOTE) atomicOr((unsigned*)(rem + (i & ~3u)), 1u << (8 * (i & 3u)));
    else ((volatile uint8_t*)own)[i] = 1;
}
__device__ __forceinline__ void pair_notify(unsigned long long nb, uint8_t* own, uint8_t* rem) {
    const unsigned lo = (unsigned)nb, hi = (unsigned)(nb >> 32);
    pair_set(own, rem, lo & 0xFFFFu);
    pair_set(own, rem, lo >> 16);
    pair_set(own, rem, hi & 0xFFFFu);
    pair_set(own, rem, (hi >> 16) & 0x7FFFu);
}
// the rest of a slow row (> SLOTS intra-pair neighbours): walk the global row
__device__ __noinline__ int pair_pull_slow(const int* own, const int* rem, const int32_t* __restrict__ ptr,
                                           const int32_t* __restrict__ adj, int pbase, int cnt, int half, int gv,
                                           int val) {
    for (int e = __ldg(ptr + gv), ee = __ldg(ptr + gv + 1); e < ee; e++) {
        const int w = __ldg(adj + e) - pbase;
        if ((unsigned)w < (unsigned)cnt) val = max(val, ((const volatile int*)((w / PACK_TT) == half ? own : rem))[w % PACK_TT]);
    }
    return val;
}
__device__ __noinline__ void pair_notify_slow(uint8_t* own, uint8_t* rem, const int32_t* __restrict__ ptr,
                                              const int32_t* __restrict__ adj, int pbase, int cnt, int half, int gv) {
    for (int e = __ldg(ptr + gv), ee = __ldg(ptr + gv + 1); e < ee; e++) {
        const int w = __ldg(adj + e) - pbase;
        if ((unsigned)w < (unsigned)cnt) {
            const unsigned i = (unsigned)(w % PACK_TT);
            if ((w / PACK_TT) == half) ((volatile uint8_t*)own)[i] = 1;
            else atomicOr((unsigned*)(rem + (i & ~3u)), 1u << (8 * (i & 3u)));
        }
    }
}

static __global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(PACK_TH, 2)
k_prop_cluster(WGraph g, int32_t* __restrict__ cin, int32_t* __restrict__ cout, const unsigned long long* __restrict__ pnin,
               const unsigned long long* __restrict__ pnout, const int2* __restrict__ ext, const int* __restrict__ ext_cnt,
               DevCounters* __restrict__ dc, AsyncQ Q, int claim) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ unsigned s_fin[PACK_TH + 1], s_fout[PACK_TH + 1];
    __shared__ int s_set[MSET];
    __shared__ int s_claim[CLAIM_MAX], s_nclaim;
    __shared__ uint8_t s_seen[CLAIM_MAX];
    __shared__ int s_any[2];
    __shared__ unsigned long long s_acc[3];
    __shared__ __align__(8) unsigned long long s_bar;
    cg::cluster_group cl = cg::this_cluster();
    const int rank = (int)cl.block_rank();
    const int tid = threadIdx.x;
    int* s_in = (int*)smem_raw;
    int* s_out = s_in + PACK_TT + 4;
    unsigned long long* s_nin = (unsigned long long*)(s_out + PACK_TT + 4);
    unsigned long long* s_nout = s_nin + PACK_TT;
    // the partner's arrays (DSMEM)
    int* r_in = cl.map_shared_rank(s_in, rank ^ 1);
    int* r_out = cl.map_shared_rank(s_out, rank ^ 1);
    uint8_t* r_fin = (uint8_t*)cl.map_shared_rank(s_fin, rank ^ 1);
    uint8_t* r_fout = (uint8_t*)cl.map_shared_rank(s_fout, rank ^ 1);
    int* r_claim = cl.map_shared_rank(s_claim, 1);
    int* r_nclaim = cl.map_shared_rank(&s_nclaim, 1);
    uint8_t* r_seen = cl.map_shared_rank(s_seen, 1);
    int* r_any = cl.map_shared_rank(s_any, rank ^ 1);
    const int npair = (g.na + PAIR_TT - 1) / PAIR_TT;
    if (tid == 0) {
        s_in[PACK_TT] = 0; s_out[PACK_TT] = 0; s_acc[0] = s_acc[1] = s_acc[2] = 0;
        mbar_init(&s_bar, 1);
    }
    unsigned phase = 0;
    volatile unsigned long long* ctr = Q.ctr;
    long long t0 = clock64();
    cl.sync();
    const int v0 = tid * VPT;
    for (;;) {
        // ---- rank 0, warp 0 claims a run of pair tiles and hands it to rank 1
        if (rank == 0 && tid < 32) {
            const int lane = tid;
            int got = 0, stop = 0;
            for (unsigned miss = 0;; miss += claim) {
                unsigned long long pos = 0;
                if (lane == 0) {
                    const unsigned long long pend = ctr[AQ_PEND], halt = ctr[AQ_STOP];
                    pos = atomicAdd(Q.ctr + AQ_CUR, (unsigned long long)claim);
                    stop = (pend == 0 || halt) ? 1 : 0;
                }
                if (__shfl_sync(FULL, stop, 0)) break;
                pos = __shfl_sync(FULL, pos, 0) + (unsigned)lane;
                bool mine = false;
                int c = 0, seen = 0;
                if (lane < claim) {
                    const unsigned long long k = pos / (unsigned)npair;
                    const int off = (int)(pos - k * (unsigned)npair);
                    c = (k & 1) ? npair - 1 - off : off;
                    const int st = ((volatile int*)Q.tstate)[c];
                    seen = ((volatile uint8_t*)Q.tseen)[c];
                    mine = st == 1 && atomicCAS(Q.tstate + c, 1, 2) == 1;
                }
                const unsigned m = __ballot_sync(FULL, mine);
                if (mine) {
                    const int slot = __popc(m & ((1u << lane) - 1));
                    s_claim[slot] = c;
                    s_seen[slot] = (uint8_t)seen;
                    r_claim[slot] = c;
                    r_seen[slot] = (uint8_t)seen;
                    if (!seen) Q.tseen[c] = 1;
                }
                if (m) { got = __popc(m); break; }
                if (miss >= (unsigned)npair) {
                    __nanosleep(256);
                    if (lane == 0 && clock64() - t0 > (1ll << 36)) {
                        atomicExch(&dc->err, 3);
                        atomicExch(Q.ctr + AQ_STOP, 1ull);
                    }
                }
            }
            if (lane == 0) {
                s_nclaim = got;
                *r_nclaim = got;
                s_acc[2] += (unsigned long long)got;
                if (got) t0 = clock64();
            }
            __threadfence();
        }
        cl.sync();                                              // the run is in both CTAs
        const int nclaim = s_nclaim;
        if (nclaim == 0) break;
        for (int j = 0; j < nclaim; j++) {
            const int pt = s_claim[j], full = s_seen[j] == 0;
            const int pbase = pt * PAIR_TT, pcnt = min(PAIR_TT, g.na - pbase);
            const int hbase = pbase + rank * PACK_TT;           // this CTA's half
            const int cnt = max(0, min(PACK_TT, pcnt - rank * PACK_TT));
            const int ne = __ldg(ext_cnt + pt);
            const int2* E = ext + (int64_t)__ldg(g.optr + pbase) + __ldg(g.iptr + pbase);
            for (int i = tid; i < MSET; i += PACK_TH) s_set[i] = -1;
            // ---- step 1: pack rows (bulk copy), own values, cut-edge pulls of own vertices
            if (tid == 0) pack_issue(pnin, pnout, 2 * pt + rank, s_nin, s_nout, &s_bar);   // this half's rows
            int x0[VPT], y0[VPT];
#pragma unroll
            for (int k = 0; k < VPT; k++) {
                x0[k] = v0 + k < cnt ? ld_cg(cin + hbase + v0 + k) : 0;
                y0[k] = v0 + k < cnt ? ld_cg(cout + hbase + v0 + k) : 0;
                s_in[v0 + k] = x0[k];
                s_out[v0 + k] = y0[k];
            }
            if (tid == 0 && cnt > 0) {
                s_acc[0] += (unsigned long long)cnt;
                s_acc[1] += (unsigned long long)(__ldg(g.optr + hbase + cnt) - __ldg(g.optr + hbase));
            }
            __syncthreads();
            for (int i = tid; i < ne; i += PACK_TH) {
                const int2 e = __ldg(E + i);
                const int v = e.y & 0x7FFF;
                if (v / PACK_TT != rank) continue;
                int* sig = (e.y & EXT_DIR) ? s_out : s_in;
                const int val = ld_cg(((e.y & EXT_DIR) ? cout : cin) + e.x);
                if (val > ((volatile int*)sig)[v % PACK_TT]) atomicMax(sig + v % PACK_TT, val);
            }
            __syncthreads();                                    // every cut-edge pull before the flags
            mbar_wait(&s_bar, phase);
            phase ^= 1u;
            unsigned fin = 0, fout = 0;
#pragma unroll
            for (int k = 0; k < VPT; k++) {
                if (v0 + k >= cnt) continue;
                if (full || s_in[v0 + k] > x0[k]) fin |= 1u << (8 * k);
                if (full || s_out[v0 + k] > y0[k]) fout |= 1u << (8 * k);
            }
            s_fin[tid] = full ? fin : 0u;
            s_fout[tid] = full ? fout : 0u;
            cl.sync();                                          // both halves loaded and flagged
            if (!full && (fin | fout)) {
#pragma unroll
                for (int k = 0; k < VPT; k++) {
                    const int v = v0 + k;
                    if ((fin >> (8 * k)) & 0xFF) {
                        pair_notify(s_nout[v], (uint8_t*)s_fin, r_fin);
                        if (s_nout[v] & SLOW_MARK) pair_notify_slow((uint8_t*)s_fin, r_fin, g.optr, g.oadj, pbase, pcnt, rank, hbase + v);
                    }
                    if ((fout >> (8 * k)) & 0xFF) {
                        pair_notify(s_nin[v], (uint8_t*)s_fout, r_fout);
                        if (s_nin[v] & SLOW_MARK) pair_notify_slow((uint8_t*)s_fout, r_fout, g.iptr, g.iadj, pbase, pcnt, rank, hbase + v);
                    }
                }
                fence_cluster();
            }
            cl.sync();
            // ---- step 2: drain both halves; rounds end with a cluster-wide OR of "worked"
            for (int round = 0;; round++) {
                int worked = 0;
                for (;;) {
                    const unsigned wi = ((volatile unsigned*)s_fin)[tid], wo = ((volatile unsigned*)s_fout)[tid];
                    const unsigned items = gather4(wi) | (gather4(wo) << 4);
                    if (!__any_sync(FULL, items != 0)) break;
                    if (items) {
                        worked = 1;
                        const int bit = __ffs(items) - 1;
                        const int v = v0 + (bit & 3);
                        const unsigned keep = ~(0xFFu << (8 * (bit & 3)));
                        if (bit & 4) {
                            atomicAnd(s_fout + tid, keep);
                            fence_cluster();
                            const unsigned long long src = s_nout[v];
                            const int old = ((volatile int*)s_out)[v];
                            int val = pair_pull(s_out, r_out, src, old);
                            if (src & SLOW_MARK) val = pair_pull_slow(s_out, r_out, g.optr, g.oadj, pbase, pcnt, rank, hbase + v, val);
                            if (val > old) {
                                ((volatile int*)s_out)[v] = val;
                                fence_cluster();
                                pair_notify(s_nin[v], (uint8_t*)s_fout, r_fout);
                                if (s_nin[v] & SLOW_MARK) pair_notify_slow((uint8_t*)s_fout, r_fout, g.iptr, g.iadj, pbase, pcnt, rank, hbase + v);
                            }
                        } else {
                            atomicAnd(s_fin + tid, keep);
                            fence_cluster();
                            const unsigned long long src = s_nin[v];
                            const int old = ((volatile int*)s_in)[v];
                            int val = pair_pull(s_in, r_in, src, old);
                            if (src & SLOW_MARK) val = pair_pull_slow(s_in, r_in, g.iptr, g.iadj, pbase, pcnt, rank, hbase + v, val);
                            if (val > old) {
                                ((volatile int*)s_in)[v] = val;
                                fence_cluster();
                                pair_notify(s_nout[v], (uint8_t*)s_fin, r_fin);
                                if (s_nout[v] & SLOW_MARK) pair_notify_slow((uint8_t*)s_fin, r_fin, g.optr, g.oadj, pbase, pcnt, rank, hbase + v);
                            }
                        }
                    }
                    __syncwarp();
                }
                // "worked" of both CTAs: each writes its own word, the cluster barrier publishes
                // it (and every remote flag set before it); words alternate by round parity,
                // so a word is rewritten only after the next barrier
                const int w = __syncthreads_or(worked);
                if (tid == 0) s_any[round & 1] = w;
                cl.sync();
                const int any = ((volatile int*)s_any)[round & 1] | ((volatile int*)r_any)[round & 1];
                if (!any) break;
            }
            // ---- step 3: write back this half, mark the pair tiles of raised cut-edge ends
            unsigned rin = 0, rout = 0;
#pragma unroll
            for (int k = 0; k < VPT; k++) {
                if (v0 + k >= cnt) continue;
                const int gi = hbase + v0 + k;
                const int xv = s_in[v0 + k], yv = s_out[v0 + k];
                if (xv > ld_cg(cin + gi)) { __stcg(cin + gi, xv); rin |= 1u << (8 * k); }
                if (yv > ld_cg(cout + gi)) { __stcg(cout + gi, yv); rout |= 1u << (8 * k); }
            }
            const int anyr = __syncthreads_or((int)(rin | rout));
            if (anyr) {
                s_fin[tid] = rin;
                s_fout[tid] = rout;
                __syncthreads();
                const uint8_t* bi = (const uint8_t*)s_fin;
                const uint8_t* bo = (const uint8_t*)s_fout;
                MarkSet mark{s_set, Q};
                for (int i = tid; i < ne; i += PACK_TH) {
                    const int2 e = __ldg(E + i);
                    const int v = e.y & 0x7FFF;
                    if (v / PACK_TT != rank) continue;
                    if (((e.y & EXT_DIR) ? bi[v % PACK_TT] : bo[v % PACK_TT]) != 0) mark(e.x / PAIR_TT);
                }
            }
            __threadfence();
            __syncthreads();
            for (int i = tid; i < MSET; i += PACK_TH)
                if (s_set[i] >= 0) aq_mark(Q, s_set[i]);
            __threadfence();
            cl.sync();                                          // both CTAs' marks before the finish
            if (rank == 0 && tid == 0) {
                aq_finish(Q, pt);
            }
        }
    }
    if (tid == 0) {
        if (s_acc[0]) atomicAdd(&dc->visit_v, s_acc[0]);
        if (s_acc[1]) atomicAdd(&dc->visit_e, s_acc[1]);
        if (s_acc[2] && rank == 0) atomicAdd(&dc->passes, s_acc[2]);
    }
    cl.sync();                                                  // no CTA leaves while its smem is mapped
}

}  // namespace eclscc
