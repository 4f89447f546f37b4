// common.cuh -- shared device helpers and the working-graph layout of the ECL-SCC path.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace eclscc {

constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr int WARP = 32;
constexpr int HEAVY = 32;      // rows longer than this are processed by a whole warp
constexpr int RING = 64;       // ring of per-pass "changed" words (Phase-2 driver)

// Working graph after an edge removal (the surviving edges, here as a compacted
// CSR + CSC pair over the ACTIVE vertices -- those that still have a live edge), in local
// numbering: local i in [0, na) is vertex act[i] (act == nullptr: identity, the input)
//   out-edges of i: oadj[optr[i] .. optr[i+1])  (local destination indices)
//   in-edges  of i: iadj[iptr[i] .. iptr[i+1])  (local source indices)
struct WGraph {
    const int32_t* act;
    const int32_t* optr;
    const int32_t* oadj;
    const int32_t* iptr;
    const int32_t* iadj;
    int32_t na;
    const int2* sig2;    // Phase 3 of power-law graphs: (v_in, v_out) interleaved, one gather per
                         // far end in keep(); nullptr: the separate cin / cout arrays
    const int32_t* min_in;   // ECL_SCC_FOUR_SIG: the minimum signatures, stored mirrored
    const int32_t* min_out;  // (INT32_MAX - priority) so Phase 2 propagates them with max;
                             // nullptr: the two-signature method
    const int32_t* hpos;     // partitioned mode (halo.cuh): position of each local vertex in the
                             // halo H, or -1; nullptr: single GPU
    const int32_t* slot;     // ECL_SCC_COMPRESS / ECL_SCC_RAISE: local index of the vertex with
                             // priority p (the vertices of the current working graph)
    int compress, raise_;    // path compression / the sound P:190 variant switched on
};
// the minimum signatures propagate as maxima of mirrored priorities (all >= 0, so the
// pack kernels' sentinel value 0 stays below every signature)
__host__ __device__ __forceinline__ int32_t mirror_prio(int32_t p) { return 0x7FFFFFFF - p; }

// Counters the host reads back once per outer iteration.
struct DevCounters {
    int4 totals;                     // after a compaction scan: (na', m_out', m_in', edges kept
                                     // by Phase 3 before trim)
    unsigned long long passes;       // Phase-2 passes that did work
    int nchunks;                     // heavy-row chunks of the current working graph
    int err;                         // validation error
    int grand1;                      // scratch total of an int32 scan
    int changed[RING];               // per-pass changed words
    unsigned long long prof[8];      // ECL_PROF builds: kernel event counters (prof[0] also: empty level-tile visits)
    unsigned long long visit_v;      // Phase 2: vertices of visited tiles (all passes)
    unsigned long long visit_e;      // Phase 2: out-edges of visited tiles (each edge once)
    unsigned long long heavy_e;      // Phase 2: edges reduced by k_prop_heavy
    unsigned long long local_e;      // ingest: short-row edges whose ends share a 2048-ID range
    int pack_bad;                    // compaction: the scatter could not write the tile pack
    int maxdeg;                      // ingest: the longest row of the input, CSR or CSC
};

// Internal vertex priorities (reading 16).  The signatures propagate
// pi(v), a keyed bijection of [0, n): a 4-round Feistel network on 2*half >= log2(n) bits
// with cycle walking.  With ids == false pi is the identity (the paper's raw IDs).
struct Prio {
    uint32_t n, half, mask, ids;
    uint32_t key[4];
};
__host__ __device__ __forceinline__ uint32_t prio_hash(uint32_t x) {
    x *= 0x9E3779B1u;
    x ^= x >> 15;
    x *= 0x85EBCA77u;
    x ^= x >> 13;
    return x;
}
__host__ __device__ __forceinline__ uint32_t prio_of(const Prio& P, uint32_t v) {
    if (P.ids) return v;
    uint32_t x = v;
    do {
        uint32_t L = x >> P.half, R = x & P.mask;
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const uint32_t nl = R;
            R = L ^ (prio_hash(R ^ P.key[r]) & P.mask);
            L = nl;
        }
        x = (L << P.half) | R;
    } while (x >= P.n);
    return x;
}
inline Prio make_prio(uint32_t n, bool ids) {
    Prio P{};
    P.n = n;
    P.ids = ids ? 1u : 0u;
    uint32_t bits = 1;
    while (bits < 32 && (1ull << bits) < (unsigned long long)n) bits++;
    P.half = (bits + 1) / 2;
    P.mask = (1u << P.half) - 1u;
    const uint32_t keys[4] = {0x3C6EF372u, 0xA54FF53Au, 0x510E527Fu, 0x9B05688Cu};
    for (int r = 0; r < 4; r++) P.key[r] = keys[r];
    return P;
}

__device__ __forceinline__ int ld_cg(const int32_t* p) { return __ldcg(p); }
__device__ __forceinline__ int ld_vol(const int* p) { return *(volatile const int*)p; }

// full-warp reductions: one REDUX instruction each (sm_80+) instead of five shuffle rounds
__device__ __forceinline__ int warp_max(int v) { return __reduce_max_sync(FULL, v); }
__device__ __forceinline__ int warp_sum(int v) { return __reduce_add_sync(FULL, v); }
// inclusive scan over the warp
__device__ __forceinline__ int warp_incl_scan(int v, int lane) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(FULL, v, o);
        if (lane >= o) v += t;
    }
    return v;
}

}  // namespace eclscc
