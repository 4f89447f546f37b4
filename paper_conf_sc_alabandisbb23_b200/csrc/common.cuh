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
};

// Counters the host reads back once per outer iteration.
struct DevCounters {
    int4 totals;                     // after a compaction scan: (na', m_out', m_in', 0)
    unsigned long long kept;         // edges kept by Phase 3 (before trim)
    unsigned long long passes;       // Phase-2 passes that did work
    int nchunks;                     // heavy-row chunks of the current working graph
    int err;                         // validation error
    int grand1;                      // scratch total of an int32 scan
    int changed[RING];               // per-pass changed words
};

__device__ __forceinline__ int ld_cg(const int32_t* p) { return __ldcg(p); }
__device__ __forceinline__ int ld_vol(const int* p) { return *(volatile const int*)p; }

__device__ __forceinline__ int warp_max(int v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(FULL, v, o));
    return v;
}
__device__ __forceinline__ int warp_sum(int v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}
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
