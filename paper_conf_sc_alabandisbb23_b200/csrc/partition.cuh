// partition.cuh -- helpers of the edge-partitioned (multi-GPU) mode: validation of a rank's
// rows and the emulated all-reduce (the algorithm itself: halo.cuh, run_halo in driver.cu).
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
