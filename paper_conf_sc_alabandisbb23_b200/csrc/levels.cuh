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
#pragma once
#include "common.cuh"

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
};

// rows longer than LV_LIGHT edges are walked by the whole warp (power-law hubs)
constexpr int LV_LIGHT = 16;

static __global__ void k_lv_count(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                  const int32_t* __restrict__ lab, int32_t* __restrict__ indeg,
                                  int32_t* __restrict__ msize, int* __restrict__ err) {
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
        {   // member counts: one atomic per label and warp (a giant SCC is in most lanes)
            const unsigned grp = __match_any_sync(FULL, L);
            if (L >= 0 && lane == __ffs(grp) - 1) atomicAdd(msize + L, __popc(grp));
        }
        const bool light = L >= 0 && ee - eb <= LV_LIGHT;
        if (light)
            for (int e = eb; e < ee; e++) {
                const int Lw = __ldg(lab + __ldg(ci + e));
                if ((unsigned)Lw >= (unsigned)n) *err = 1;
                else if (Lw != L) atomicAdd(indeg + Lw, 1);
            }
        unsigned hv = __ballot_sync(FULL, L >= 0 && !light);
        while (hv) {
            const int src = __ffs(hv) - 1;
            hv &= hv - 1;
            const int sb = __shfl_sync(FULL, eb, src), se = __shfl_sync(FULL, ee, src), sL = __shfl_sync(FULL, L, src);
            for (int e = sb + lane; e < se; e += WARP) {
                const int Lw = __ldg(lab + __ldg(ci + e));
                if ((unsigned)Lw >= (unsigned)n) *err = 1;
                else if (Lw != sL) atomicAdd(indeg + Lw, 1);
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

}  // namespace eclscc
