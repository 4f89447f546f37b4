// halo.cuh -- kernels of the edge-partitioned mode, "halo" form.
//
// Rank r owns source rows [rb, re): the out-edges u -> w of its vertices (global IDs).  Its
// LOCAL graph is those edges over local vertices = the owned ones (local 0..nloc-1, in ID
// order) followed by the ghosts (destinations owned elsewhere, nloc.., in ID order), and it
// runs the single-GPU machinery unchanged (tile packs, k_prop_async, compaction) with
// global priorities (the local -> global map plays the role of the storage-order map).
// Every edge lives on exactly one rank; a vertex held by several ranks (a ghost somewhere:
// the halo H) has one signature copy per holder.  Copies are combined by MAX:
//   * Phase 2 (Alg. 1 l.7-14): each rank relaxes its edges to a LOCAL fixed point; every
//     raise of a halo copy is pushed into the exchange buffer of every rank (remote atomic
//     max over NVLink peer memory, or one multimem reduction through the NVSwitch) by the
//     propagation kernel itself, tile by tile (HaloPush).  After a barrier each rank folds
//     the buffer into its copies; a copy that rose re-opens its tile (a full visit).  When no
//     rank injected anything every copy equals the maximum and every edge satisfies the
//     fixed-point inequality on its rank: the global fixed point (reading 12).
//   * Trim-1 needs global degrees of halo vertices: a SUM exchange of the kept
//     degrees over H per iteration.
//   * Phase 3 is local: both ends of an edge are on its rank, with equal copies.
//   * An unfinished halo vertex stays in a rank's working graph even without local edges
//     (its edges may live elsewhere); finished vertices leave on every holder at once.
// Exchange volume per round: |H| signature pairs (the slab faces), not 2n.
#pragma once
#include "common.cuh"

namespace eclscc {

// where the propagation kernel pushes raised halo copies (hpos == nullptr: not partitioned)
constexpr int HALO_MAX_PEERS = 8;
struct HaloPush {
    const int32_t* hpos;                  // per local vertex: position in H, or -1
    int32_t* peer[HALO_MAX_PEERS];        // every rank's exchange buffer ([2p] in, [2p+1] out)
    int32_t* mc;                          // multimem (NVLS multicast) address of the buffers, or nullptr
    int np;
    int sys;                              // peers on other GPUs: system-scope atomics + fence
};

__device__ __forceinline__ void halo_push_one(const HaloPush& H, int64_t off, int val) {
    if (H.mc) {
        asm volatile("multimem.red.relaxed.sys.global.max.s32 [%0], %1;" ::"l"(H.mc + off), "r"(val) : "memory");
        return;
    }
    for (int k = 0; k < H.np; k++) {
        if (H.sys) atomicMax_system(H.peer[k] + off, val);
        else atomicMax(H.peer[k] + off, val);
    }
}

// ------------------------------------------------------------------ ingest
// destinations outside the owned rows are ghosts: mark them (global-indexed)
static __global__ void k_halo_mark_ghosts(int64_t m, const int32_t* __restrict__ ci, int32_t rb, int32_t re,
                                          int32_t* __restrict__ gmark) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x) {
        const int w = __ldg(ci + e);
        if (w < rb || w >= re) gmark[w] = 1;
    }
}
// local -> global map: owned rows first, then the ghosts in ID order (gidx = exclusive scan
// of the marks); halo membership (hb) of every local vertex becomes its position in H
static __global__ void k_halo_l2g(int32_t n, int32_t rb, int32_t re, const int32_t* __restrict__ gmark,
                                  const int32_t* __restrict__ gidx, int32_t* __restrict__ l2g) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < n; w += (int64_t)gridDim.x * blockDim.x) {
        if (w >= rb && w < re) l2g[w - rb] = (int32_t)w;
        else if (gmark[w]) l2g[(re - rb) + gidx[w]] = (int32_t)w;
    }
}
static __global__ void k_halo_local_csr(int32_t nloc, int32_t ng, int64_t m, const int32_t* __restrict__ rp,
                                        const int32_t* __restrict__ ci, int32_t rb, int32_t re,
                                        const int32_t* __restrict__ gidx, int32_t* __restrict__ lrp,
                                        int32_t* __restrict__ lci) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t e = t0; e < m; e += stride) {
        const int w = __ldg(ci + e);
        lci[e] = (w >= rb && w < re) ? w - rb : nloc + __ldg(gidx + w);
    }
    for (int64_t i = t0; i <= (int64_t)nloc + ng; i += stride) lrp[i] = i <= nloc ? __ldg(rp + i) : (int32_t)m;
}
// position in H of every local vertex (hb: halo membership summed over ranks, hposg its
// exclusive scan over the global IDs)
static __global__ void k_halo_hpos(int32_t nl, const int32_t* __restrict__ l2g, const int32_t* __restrict__ hb,
                                   const int32_t* __restrict__ hposg, int32_t* __restrict__ hpos) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nl; i += (int64_t)gridDim.x * blockDim.x) {
        const int w = __ldg(l2g + i);
        hpos[i] = __ldg(hb + w) > 0 ? __ldg(hposg + w) : -1;
    }
}
static __global__ void k_nonzero(int64_t n, const int32_t* __restrict__ in, int32_t* __restrict__ out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        out[v] = in[v] != 0;
}

// ------------------------------------------------------------------ per iteration
// kept degrees of the halo copies -> the SUM buffer (entries this rank does not hold stay 0)
static __global__ void k_halo_deg_pack(int32_t na, const int32_t* __restrict__ hpos, const int2* __restrict__ kio,
                                       int32_t* __restrict__ hdeg) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < na; i += (int64_t)gridDim.x * blockDim.x) {
        const int p = hpos[i];
        if (p >= 0) {
            const int2 k = kio[i];
            hdeg[2 * (int64_t)p] = k.x;
            hdeg[2 * (int64_t)p + 1] = k.y;
        }
    }
}
static __global__ void k_halo_deg_apply(int32_t na, const int32_t* __restrict__ hpos, const int32_t* __restrict__ hdeg,
                                        int2* __restrict__ kio) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < na; i += (int64_t)gridDim.x * blockDim.x) {
        const int p = hpos[i];
        if (p >= 0) kio[i] = make_int2(hdeg[2 * (int64_t)p], hdeg[2 * (int64_t)p + 1]);
    }
}
// the local phase of a non-asynchronous Phase 2 (pass kernels): push every halo copy
static __global__ void k_halo_push(int32_t na, const int32_t* __restrict__ cin, const int32_t* __restrict__ cout,
                                   HaloPush H) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < na; i += (int64_t)gridDim.x * blockDim.x) {
        const int p = H.hpos[i];
        if (p >= 0) {
            halo_push_one(H, 2 * (int64_t)p, cin[i]);
            halo_push_one(H, 2 * (int64_t)p + 1, cout[i]);
        }
    }
    if (H.sys) __threadfence_system();
}
// fold the exchange buffer into the local copies.  A copy that rose re-opens its own tile for
// a full visit (its intra-tile dependents re-pull) and the tiles of its cut-edge dependents
// (a raised v_in reaches the out-neighbours, a raised v_out the in-neighbours; their visit's
// cut-edge pulls see the new value).  Asynchronous Phase 2: tile state 0 -> 1, pending++;
// pass mode: dirty flags (pass 0 visits them fully).
__device__ __forceinline__ void halo_open(int t, int* tstate, unsigned long long* pending, uint8_t* dirty) {
    if (tstate && atomicCAS(tstate + t, 0, 1) == 0) atomicAdd(pending, 1ull);
    if (dirty) dirty[t] = 1;
}
static __global__ void k_halo_apply(WGraph g, const int32_t* __restrict__ hbuf, int32_t* __restrict__ cin,
                                    int32_t* __restrict__ cout, int* __restrict__ tstate, uint8_t* __restrict__ tseen,
                                    unsigned long long* __restrict__ pending, uint8_t* __restrict__ dirty, int tile,
                                    int* __restrict__ injected) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < g.na; i += (int64_t)gridDim.x * blockDim.x) {
        const int p = g.hpos[i];
        if (p < 0) continue;
        const int x = hbuf[2 * (int64_t)p], y = hbuf[2 * (int64_t)p + 1];
        const bool ui = x > cin[i], uo = y > cout[i];
        if (!(ui | uo)) continue;
        if (ui) cin[i] = x;
        if (uo) cout[i] = y;
        *injected = 1;
        const int t = (int)(i / tile);
        if (tseen) tseen[t] = 0;
        halo_open(t, tstate, pending, dirty);
        if (ui)
            for (int e = g.optr[i], ee = g.optr[i + 1]; e < ee; e++) {
                const int tw = g.oadj[e] / tile;
                if (tw != t) halo_open(tw, tstate, pending, dirty);
            }
        if (uo)
            for (int e = g.iptr[i], ee = g.iptr[i + 1]; e < ee; e++) {
                const int tu = g.iadj[e] / tile;
                if (tu != t) halo_open(tu, tstate, pending, dirty);
            }
    }
}
// the working graph's remaining vertices at global termination: unfinished and edgeless
// everywhere, so singletons (rule R2); only the owner writes the label
static __global__ void k_halo_final(int32_t na, const int32_t* __restrict__ act, const int32_t* __restrict__ l2g,
                                    int32_t rb, int32_t re, int32_t* __restrict__ lab) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < na; i += (int64_t)gridDim.x * blockDim.x) {
        const int v = l2g[act ? act[i] : (int)i];
        if (v >= rb && v < re) lab[v] = v;
    }
}
static __global__ void k_fill(int64_t n, int32_t* __restrict__ a, int32_t v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) a[i] = v;
}

}  // namespace eclscc
