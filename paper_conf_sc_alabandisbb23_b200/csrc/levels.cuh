// levels.cuh -- the sweep schedule after SCC detection: levels of the SCC condensation.
//
// A transport sweep for one ordinate traverses the induced graph "starting from nodes with no
// incoming edges"; once the SCCs are known the sweep proceeds over the condensation, a
// DAG whose depth the paper tabulates per mesh (Table 2, "DAG depth").  level(C) = the length
// of the longest condensation path ending in SCC C (sources: 0); the SCCs of one level can be
// swept concurrently.
//
// GPU plan (Kahn's algorithm, level-synchronous, in one cooperative launch):
//   k_lv_count   per label: member count and in-degree from other SCCs (edge-parallel rows)
//   scan         member offsets;  k_lv_fill: members grouped by label
//   k_lv_init    source SCCs (in-degree 0) form frontier 0, as chunk items of <= 8 members
//   k_lv_run     round l: one lane per chunk item (mesh SCCs are mostly singletons: a warp
//                per item would idle 31 lanes; rows longer than 16 edges are walked by the
//                whole warp), its members' out-edges into other SCCs
//                decrement their in-degree; the decrement that reaches 0 makes
//                that SCC level l+1 and appends its chunk items to the next frontier; a grid
//                barrier ends the round (longest-path levels: an SCC is ready exactly one round
//                after its deepest predecessor)
//   k_lv_apply   levels_out[v] = level of label(v); depth = max level + 1
// SCCs never reached mean the labels induce a cycle (not the SCC partition): ERANGE.
//
// Tile mode (the default when the labels' cross edges mostly stay inside 2048-node tiles,
// e.g. meshes): the same Kahn rule, run asynchronously per tile by the Phase-2 tile queue
// instead of in global rounds (k_lk_*, below).  Kahn's rounds remain for low-locality graphs
// (power-law: depth ~8, few rounds) and behind ECL_SCC_NO_ASYNC.
#pragma once
#include "common.cuh"
#include "pack.cuh"    // the tile queue (AsyncQ, aq_claim, MarkSet) of the tile mode

namespace eclscc {

// grid barrier among the co-resident CTAs of a cooperative launch (one CTA: a block barrier)
__device__ __forceinline__ void grid_bar(unsigned* bar, int G) {
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

struct LvCtl {
    unsigned bar[2];         // grid barrier
    int size[3];             // frontier sizes, round % 3
    int nscc;                // labels in use
    int reached;             // SCCs that got a level
    int depth;               // max level + 1
    int rounds;
    int err;                 // label out of range
    int maxodeg;             // tile mode: the largest cross out-degree of a node
    unsigned long long intra, cross;   // tile mode: cross edges inside one tile / between tiles
};

// rows longer than LV_LIGHT edges are walked by the whole warp (power-law hubs)
constexpr int LV_LIGHT = 16;

// odeg (optional, the tile mode): cross out-edges per label, and ctl_intra[0 / 1] the cross
// edges inside one 2048-ID tile / between tiles
static __global__ void k_lv_count(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                  const int32_t* __restrict__ lab, int32_t* __restrict__ indeg,
                                  int32_t* __restrict__ msize, int* __restrict__ err, int32_t* __restrict__ odeg,
                                  unsigned long long* __restrict__ ctl_intra) {
    const int lane = threadIdx.x & 31;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t u0 = (int64_t)blockIdx.x * blockDim.x; u0 < n; u0 += stride) {   // warp-uniform trip count
        const int64_t u = u0 + threadIdx.x;
        int L = -1, eb = 0, ee = 0;
        if (u < n) {
            L = __ldg(lab + u);
            if ((unsigned)L >= (unsigned)n) { *err = 1; L = -1; }
            else {
                eb = __ldg(rp + u);
                ee = __ldg(rp + u + 1);
            }
        }
        const unsigned grp = __match_any_sync(FULL, L);
        // member counts: one atomic per label and warp (a giant SCC is in most lanes)
        if (L >= 0 && lane == __ffs(grp) - 1) atomicAdd(msize + L, __popc(grp));
        const bool light = L >= 0 && ee - eb <= LV_LIGHT;
        int cross = 0, near = 0;                           // near: cross edges inside one 2048-ID tile
        if (light)
            for (int e = eb; e < ee; e++) {
                const int Lw = __ldg(lab + __ldg(ci + e));
                if ((unsigned)Lw >= (unsigned)n) *err = 1;
                else if (Lw != L) { atomicAdd(indeg + Lw, 1); cross++; near += (Lw >> 11) == (L >> 11); }
            }
        unsigned hv = __ballot_sync(FULL, L >= 0 && !light);
        while (hv) {
            const int src = __ffs(hv) - 1;
            hv &= hv - 1;
            const int sb = __shfl_sync(FULL, eb, src), se = __shfl_sync(FULL, ee, src), sL = __shfl_sync(FULL, L, src);
            int cc = 0, nn = 0;
            for (int e = sb + lane; e < se; e += WARP) {
                const int Lw = __ldg(lab + __ldg(ci + e));
                if ((unsigned)Lw >= (unsigned)n) *err = 1;
                else if (Lw != sL) { atomicAdd(indeg + Lw, 1); cc++; nn += (Lw >> 11) == (sL >> 11); }
            }
            cc = warp_sum(cc);
            nn = warp_sum(nn);
            if (lane == src) { cross += cc; near += nn; }
        }
        if (odeg) {                                        // one atomic per label and warp
            const int t = __reduce_add_sync(grp, cross);
            if (L >= 0 && t && lane == __ffs(grp) - 1) atomicAdd(odeg + L, t);
            const int tn = __reduce_add_sync(FULL, near), tc = __reduce_add_sync(FULL, cross);
            if (lane == 0 && tc) {
                atomicAdd(&ctl_intra[0], (unsigned long long)tn);
                atomicAdd(&ctl_intra[1], (unsigned long long)(tc - tn));
            }
        }
    }
}

static __global__ void k_lv_fill(int32_t n, const int32_t* __restrict__ lab, const int32_t* __restrict__ mptr,
                                 int32_t* __restrict__ cursor, int32_t* __restrict__ memb) {
    const int lane = threadIdx.x & 31;
    for (int64_t u0 = (int64_t)blockIdx.x * blockDim.x; u0 < n; u0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t u = u0 + threadIdx.x;
        const int L = u < n ? __ldg(lab + u) : -1;
        // lanes of one label take consecutive slots with one atomic per label and warp
        const unsigned grp = __match_any_sync(FULL, L);
        const int leader = __ffs(grp) - 1;
        int at = 0;
        if (L >= 0 && lane == leader) at = atomicAdd(cursor + L, __popc(grp));
        at = __shfl_sync(FULL, at, leader);
        if (L >= 0) memb[__ldg(mptr + L) + at + __popc(grp & ((1u << lane) - 1))] = (int32_t)u;
    }
}

constexpr int LV_CHUNK = 8;      // members per frontier item
constexpr int LV_STAGE = 2048;   // ready SCCs staged per CTA and round

// append the chunk items of SCC c to a frontier
__device__ __forceinline__ void lv_push(int c, const int32_t* __restrict__ mptr, int2* __restrict__ q, int* size) {
    const int b = __ldg(mptr + c), e = __ldg(mptr + c + 1);
    const int k = (e - b + LV_CHUNK - 1) / LV_CHUNK;
    const int at = atomicAdd(size, k);
    for (int j = 0; j < k; j++) q[at + j] = make_int2(c, b + LV_CHUNK * j);
}

static __global__ void k_lv_init(int32_t n, const int32_t* __restrict__ indeg, const int32_t* __restrict__ msize,
                                 const int32_t* __restrict__ mptr, int32_t* __restrict__ lvl, int2* __restrict__ q0,
                                 LvCtl* ctl) {
    int cnt = 0, src = 0;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
        lvl[c] = -1;
        if (msize[c] == 0) continue;                   // not a label
        cnt++;
        if (indeg[c] == 0) {                           // a source SCC: level 0
            lvl[c] = 0;
            src++;
            lv_push((int)c, mptr, q0, &ctl->size[0]);
        }
    }
    cnt = warp_sum(cnt);
    src = warp_sum(src);
    if ((threadIdx.x & 31) == 0) {
        if (cnt) atomicAdd(&ctl->nscc, cnt);
        if (src) atomicAdd(&ctl->reached, src);
    }
}

static __global__ void __launch_bounds__(512) k_lv_run(const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                                       const int32_t* __restrict__ lab, const int32_t* __restrict__ mptr,
                                                       const int32_t* __restrict__ memb, int32_t* indeg, int32_t* lvl,
                                                       int2* qa, int2* qb, LvCtl* ctl) {
    const int G = gridDim.x;
    const int lane = threadIdx.x & 31;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)G * blockDim.x) >> 5;
    // SCCs made ready in a round are staged in shared memory and appended to the next
    // frontier with ONE global atomic per CTA (a single frontier counter hit by every push
    // serialised ~12k atomics per round on C4)
    __shared__ int s_list[LV_STAGE], s_off[LV_STAGE];
    __shared__ int s_nl, s_total, s_gbase;
    if (threadIdx.x == 0) { s_nl = 0; s_total = 0; }
    __syncthreads();
    int2* cur = qa;
    int2* nxt = qb;
    int reached = 0;                                  // summed once at the end (one address)
    for (int l = 0;; l++) {
        const int ncur = *(volatile int*)&ctl->size[l % 3];
        int* nsize = &ctl->size[(l + 1) % 3];
        // an out-edge u -> w of the current frontier: the last one into SCC d makes d ready
        auto relax_to = [&](int d, int c) {
            if (d != c && atomicSub(indeg + d, 1) == 1) {          // d's last predecessor edge
                lvl[d] = l + 1;
                reached++;
                const int pos = atomicAdd(&s_nl, 1);
                if (pos < LV_STAGE) s_list[pos] = d;
                else lv_push(d, mptr, nxt, nsize);                 // stage full: direct
            }
        };
        auto relax = [&](int e, int c) { relax_to(__ldg(lab + __ldg(ci + e)), c); };
        // one item per lane; light rows by their lane, rows > LV_LIGHT edges by the warp
        for (int64_t base = wid * 32; base < ncur; base += nw * 32) {
            const int64_t it = base + lane;
            int c = -1, mb = 0, me = 0;
            if (it < ncur) {
                const int2 item = __ldcg(cur + it);               // written by other SMs last round
                c = item.x;
                mb = item.y;
                me = min(mb + LV_CHUNK, __ldg(mptr + c + 1));
            }
            for (int k = 0; k < LV_CHUNK; k++) {
                const bool has = mb + k < me;
                int eb = 0, ee = 0;
                if (has) {
                    const int u = __ldg(memb + mb + k);
                    eb = __ldg(rp + u);
                    ee = __ldg(rp + u + 1);
                }
                const bool light = has && ee - eb <= LV_LIGHT;
                if (light)
                    for (int e = eb; e < ee; e += 4) {                // loads of 4 edges before use
                        int w[4], d[4];
#pragma unroll
                        for (int q = 0; q < 4; q++) w[q] = e + q < ee ? __ldg(ci + e + q) : -1;
#pragma unroll
                        for (int q = 0; q < 4; q++) d[q] = w[q] >= 0 ? __ldg(lab + w[q]) : c;
#pragma unroll
                        for (int q = 0; q < 4; q++) relax_to(d[q], c);
                    }
                unsigned hv = __ballot_sync(FULL, has && !light);
                while (hv) {
                    const int src = __ffs(hv) - 1;
                    hv &= hv - 1;
                    const int sb = __shfl_sync(FULL, eb, src), se = __shfl_sync(FULL, ee, src);
                    const int sc = __shfl_sync(FULL, c, src);
                    for (int e = sb + lane; e < se; e += WARP) relax(e, sc);
                }
                if (!__any_sync(FULL, mb + k + 1 < me)) break;
            }
        }
        __syncthreads();
        const int nl = min(s_nl, LV_STAGE);
        for (int i = threadIdx.x; i < nl; i += blockDim.x) {
            const int d = s_list[i];
            s_off[i] = atomicAdd(&s_total, (__ldg(mptr + d + 1) - __ldg(mptr + d) + LV_CHUNK - 1) / LV_CHUNK);
        }
        __syncthreads();
        if (threadIdx.x == 0) s_gbase = s_total ? atomicAdd(nsize, s_total) : 0;
        __syncthreads();
        for (int i = threadIdx.x; i < nl; i += blockDim.x) {
            const int d = s_list[i];
            const int b = __ldg(mptr + d), e = __ldg(mptr + d + 1);
            for (int j = 0, at = s_gbase + s_off[i]; b + LV_CHUNK * j < e; j++) nxt[at + j] = make_int2(d, b + LV_CHUNK * j);
        }
        __syncthreads();
        if (threadIdx.x == 0) { s_nl = 0; s_total = 0; }

        if (blockIdx.x == 0 && threadIdx.x == 0) ctl->size[(l + 2) % 3] = 0;   // read two rounds ago
        __threadfence();
        grid_bar(ctl->bar, G);
        if (*(volatile int*)&ctl->size[(l + 1) % 3] == 0) {
            if (blockIdx.x == 0 && threadIdx.x == 0) {
                ctl->depth = ncur > 0 ? l + 1 : l;
                ctl->rounds = l + 1;
            }
            break;
        }
        int2* t = cur;
        cur = nxt;
        nxt = t;
    }
    reached = warp_sum(reached);
    if (lane == 0 && reached) atomicAdd(&ctl->reached, reached);
}

static __global__ void k_lv_apply(int32_t n, const int32_t* __restrict__ lab, const int32_t* __restrict__ lvl,
                                  int32_t* __restrict__ out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        out[v] = __ldg(lvl + __ldg(lab + v));
}

// ------------------------------------------------------------------ tile mode
// Nodes are the SCCs, each identified by its label (the largest member's ID, so a node sits
// in the ID range -- the tile -- of its members).  Cross edges c -> d (d != c) form a CSR over
// nodes (cptr / cadj).  Kahn's rule per node: ready once every cross in-edge's source is
// done; level = max over them of (level + 1), sources 0.  The in-count is split: icnt (sources
// in the same 2048-node tile) is decremented in shared memory by the tile's own visits and
// persisted between them; ecnt (sources in other tiles) is decremented with a global atomic
// by the visit that finishes the source, after it folded its level into lvl_ext, and the
// decrement that reaches 0 marks the node's tile dirty.  A visit snapshots ecnt, then runs
// the tile's own Kahn in shared memory (one ready node per lane and warp round, as the
// Phase-2 drain); tiles are scheduled by the Phase-2 queue (pack.cuh AsyncQ: a node whose
// last external source finishes during a visit is picked up by the revisit that the mark
// forces).  Every node is processed once, when its level is final.  Nodes never processed
// at the fixed point lie on a cycle of the labels' condensation: ERANGE.
constexpr int LK_TT = 2048, LK_TH = 512, LK_ECAP = 4096;   // nodes per tile, threads, cached cross edges
constexpr int LK_XCAP = 2048;    // external updates of a visit batched behind one fence
struct LkState {
    const int32_t* cptr;     // [n + 1] cross edges of node c: cadj[cptr[c] .. cptr[c + 1])
    const int32_t* cadj;
    int32_t* icnt;           // [n] intra-tile in-count left (-1 once done)
    int32_t* ecnt;           // [n] external in-count left
    int32_t* lvl;            // [n] level from intra-tile sources so far; the level once done
    int32_t* lvl_ext;        // [n] level from other tiles' sources so far
    int32_t n;
};

// cross-edge lists (filled at cptr[c] + cursor) and the split in-counts
static __global__ void k_lk_fill(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                 const int32_t* __restrict__ lab, const int32_t* __restrict__ cptr,
                                 int32_t* __restrict__ ccur, int32_t* __restrict__ cadj, int32_t* __restrict__ icnt,
                                 int32_t* __restrict__ ecnt) {
    const int lane = threadIdx.x & 31;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t u0 = (int64_t)blockIdx.x * blockDim.x; u0 < n; u0 += stride) {
        const int64_t u = u0 + threadIdx.x;
        int L = -1, eb = 0, ee = 0;
        if (u < n) {
            L = __ldg(lab + u);
            eb = __ldg(rp + u);
            ee = __ldg(rp + u + 1);
        }
        auto put = [&](int c, int d) {
            cadj[__ldg(cptr + c) + atomicAdd(ccur + c, 1)] = d;
            atomicAdd((c / LK_TT == d / LK_TT ? icnt : ecnt) + d, 1);
        };
        const bool light = L >= 0 && ee - eb <= LV_LIGHT;
        if (light)
            for (int e = eb; e < ee; e++) {
                const int d = __ldg(lab + __ldg(ci + e));
                if (d != L) put(L, d);
            }
        unsigned hv = __ballot_sync(FULL, L >= 0 && !light);
        while (hv) {
            const int src = __ffs(hv) - 1;
            hv &= hv - 1;
            const int sb = __shfl_sync(FULL, eb, src), se = __shfl_sync(FULL, ee, src), sL = __shfl_sync(FULL, L, src);
            for (int e = sb + lane; e < se; e += WARP) {
                const int d = __ldg(lab + __ldg(ci + e));
                if (d != sL) put(sL, d);
            }
        }
    }
}
// node state: non-labels are done from the start; the label count and the largest cross
// out-degree (the tile mode walks a node's list by one lane)
static __global__ void k_lk_init(int32_t n, const int32_t* __restrict__ msize, const int32_t* __restrict__ cptr,
                                 int32_t* __restrict__ icnt, int32_t* __restrict__ lvl, int32_t* __restrict__ lvl_ext,
                                 LvCtl* ctl) {
    int cnt = 0, mo = 0;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
        lvl[c] = 0;
        lvl_ext[c] = 0;
        if (msize[c] == 0) { icnt[c] = -1; continue; }
        cnt++;
        mo = max(mo, cptr[c + 1] - cptr[c]);
    }
    cnt = warp_sum(cnt);
    mo = __reduce_max_sync(FULL, mo);
    if ((threadIdx.x & 31) == 0) {
        if (cnt) atomicAdd(&ctl->nscc, cnt);
        if (mo) atomicMax(&ctl->maxodeg, mo);
    }
}
static __global__ void __launch_bounds__(LK_TH, 3) k_lk_run(LkState L, DevCounters* __restrict__ dc, AsyncQ Q, int claim) {
    extern __shared__ int s_e[];                       // [LK_ECAP] the tile's cross edges
    __shared__ int s_icnt[LK_TT], s_lvl[LK_TT], s_cp[LK_TT + 1];
    __shared__ unsigned s_f[LK_TH];                    // ready flags, a byte per node
    __shared__ uint8_t s_ext0[LK_TT];                  // ecnt == 0 at the visit's start
    __shared__ int s_set[MSET];
    __shared__ int s_claim[CLAIM_MAX], s_nclaim;
    __shared__ uint8_t s_seen[CLAIM_MAX];
    __shared__ int2 s_x[LK_XCAP];                      // external updates {node, level} of the visit
    __shared__ int s_nx;
    const int tid = threadIdx.x, v0 = tid * 4;
    const int ntiles = (L.n + LK_TT - 1) / LK_TT;
    long long t0 = clock64();
    unsigned long long visits = 0, empty = 0;
    for (;;) {
        if (tid < 32) {
            const int got = aq_claim(Q, ntiles, claim, tid, s_claim, s_seen, t0, dc);
            if (tid == 0) {
                s_nclaim = got;
                visits += (unsigned long long)got;
                if (got) t0 = clock64();
            }
            __threadfence();                           // claims before the counter reads
        }
        __syncthreads();
        const int nclaim = s_nclaim;
        if (nclaim == 0) break;
        for (int j = 0; j < nclaim; j++) {
            const int tile = s_claim[j];
            const int base = tile * LK_TT, cnt = min(LK_TT, L.n - base);
            const int eb = __ldg(L.cptr + base);
            const int ne = __ldg(L.cptr + base + cnt) - eb;
            unsigned f = 0;
            int ic[4], lv[4], ec[4];                   // (lv: as stored, to write back what changed)
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const int v = v0 + k;
                ic[k] = -1; lv[k] = 0; ec[k] = 1;
                if (v < cnt) {
                    ic[k] = L.icnt[base + v];
                    lv[k] = L.lvl[base + v];
                    ec[k] = __ldcg(L.ecnt + base + v);
                }
            }
            __threadfence();                           // a zero ecnt before the lvl_ext reads: final
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const int v = v0 + k;
                int l = lv[k];
                if (v < cnt && ic[k] >= 0 && ec[k] == 0) l = max(l, __ldcg(L.lvl_ext + base + v));
                s_icnt[v] = ic[k];
                s_lvl[v] = l;
                s_ext0[v] = ec[k] == 0;
                if (ic[k] == 0 && ec[k] == 0) f |= 1u << (8 * k);
            }
            s_f[tid] = f;
            // a visit whose marks brought no node to readiness changes nothing (most revisits:
            // an external count reached 0 while intra-tile sources are still pending)
            const int nonempty = __syncthreads_or(f != 0);
            if (tid == 0 && !nonempty) empty++;
            if (nonempty) {
            for (int i = tid; i < MSET; i += LK_TH) s_set[i] = -1;
            if (tid == 0) s_nx = 0;
            for (int i = tid; i < min(ne, LK_ECAP); i += LK_TH) s_e[i] = __ldg(L.cadj + eb + i);
            for (int i = tid; i <= cnt; i += LK_TH) s_cp[i] = __ldg(L.cptr + base + i) - eb;
            __syncthreads();
            // local Kahn: a flagged node is ready; its level is final
            for (;;) {
                int worked = 0;
                for (;;) {
                    const unsigned items = gather4(((volatile unsigned*)s_f)[tid]);
                    if (!__any_sync(FULL, items != 0)) break;
                    if (items) {
                        worked = 1;
                        const int k = __ffs(items) - 1, v = v0 + k;
                        atomicAnd(s_f + tid, ~(0xFFu << (8 * k)));
                        // (the external sources' level came with the snapshot: ecnt was 0)
                        const int lv = ((volatile int*)s_lvl)[v];
                        ((volatile int*)s_icnt)[v] = -1;                  // done
                        for (int e = s_cp[v], ee = s_cp[v + 1]; e < ee; e++) {
                            const int d = e < LK_ECAP ? s_e[e] : __ldg(L.cadj + eb + e);
                            const int dl = d - base;
                            if ((unsigned)dl < (unsigned)cnt) {
                                atomicMax(s_lvl + dl, lv + 1);
                                __threadfence_block();
                                if (atomicSub(s_icnt + dl, 1) == 1 && s_ext0[dl])
                                    atomicOr(s_f + (dl >> 2), 1u << (8 * (dl & 3)));
                            } else {                                       // after the drain
                                const int at = atomicAdd(&s_nx, 1);
                                if (at < LK_XCAP) s_x[at] = make_int2(d, lv + 1);
                                else {
                                    atomicMax(L.lvl_ext + d, lv + 1);
                                    __threadfence();                       // the level before the count
                                    if (atomicSub(L.ecnt + d, 1) == 1) MarkSet{s_set, Q}(d / LK_TT);
                                }
                            }
                        }
                    }
                    __syncwarp();
                }
                if (!__syncthreads_or(worked)) break;
            }
            {                                          // the external updates: levels, one fence, counts
                const int nx = min(s_nx, LK_XCAP);
                for (int i = tid; i < nx; i += LK_TH) atomicMax(L.lvl_ext + s_x[i].x, s_x[i].y);
                __threadfence();
                __syncthreads();
                for (int i = tid; i < nx; i += LK_TH)
                    if (atomicSub(L.ecnt + s_x[i].x, 1) == 1) MarkSet{s_set, Q}(s_x[i].x / LK_TT);
            }
#pragma unroll
            for (int k = 0; k < 4; k++) {              // write back what changed
                const int v = v0 + k;
                if (v < cnt) {
                    if (s_icnt[v] != ic[k]) L.icnt[base + v] = s_icnt[v];
                    if (s_lvl[v] != lv[k]) L.lvl[base + v] = s_lvl[v];
                }
            }
            __threadfence();
            __syncthreads();
            for (int i = tid; i < MSET; i += LK_TH)
                if (s_set[i] >= 0) aq_mark(Q, s_set[i]);
            __threadfence();
            }
            __syncthreads();                           // marks (pending++) before finish
            if (tid == 0) {
                aq_finish(Q, tile);
            }
        }
        __syncthreads();                               // s_claim is rewritten next
    }
    if (tid == 0 && visits) atomicAdd(&dc->passes, visits);
    if (tid == 0 && empty) atomicAdd(&dc->prof[0], empty);    // visits that found no node ready
}
// levels_out[v] = level of label(v); depth; every label processed (else a cyclic condensation)
static __global__ void k_lk_apply(int32_t n, const int32_t* __restrict__ lab, const int32_t* __restrict__ msize,
                                  const int32_t* __restrict__ icnt, const int32_t* __restrict__ lvl,
                                  int32_t* __restrict__ out, LvCtl* ctl) {
    int dmax = 0, done = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int c = __ldg(lab + v);
        const int l = __ldg(lvl + c);
        out[v] = l;
        dmax = max(dmax, l + 1);
        if (msize[v] > 0 && icnt[v] == -1) done++;    // v is a label, processed
    }
    dmax = __reduce_max_sync(FULL, dmax);
    done = warp_sum(done);
    if ((threadIdx.x & 31) == 0) {
        if (dmax) atomicMax(&ctl->depth, dmax);
        if (done) atomicAdd(&ctl->reached, done);
    }
}

}  // namespace eclscc
