// reorder.cuh -- storage reordering of the input graph.
//
// Tiles are ranges of consecutive vertices, so their shape is whatever the caller's
// numbering makes of them.  For graphs without long rows (meshes) the library clusters the
// vertices with a multi-source BFS over in- and out-edges from pseudo-random seeds (a graph
// Voronoi partition with ~TILE vertices per cell), renumbers them cell by cell into a
// permuted CSR, and keeps orig[] so priorities and labels stay in the caller's IDs.  The
// SCC result does not depend on the storage order (the fixed points are unique), only the
// number of Phase-2 passes does.
#pragma once
#include "common.cuh"

namespace eclscc {
namespace reo {

constexpr int CELL_SHIFT = 11;        // ~2048 vertices per cell
constexpr int NOLAB = 0x7FFFFFFF;

__device__ __forceinline__ bool is_seed(int v) {
    return (prio_hash((uint32_t)v ^ 0x5BD1E995u) & ((1u << CELL_SHIFT) - 1)) == 0;
}

// one BFS level (persistent, grid-stride): every frontier vertex offers its cell to
// unclaimed neighbours (first offer wins, so the partition depends on the schedule --
// harmless: only the number of passes depends on it).  Counters rotate over three words:
// level r reads cnt[r%3], appends to cnt[(r+1)%3] and clears cnt[(r+2)%3].
static __global__ void k_bfs_level(int32_t* __restrict__ fa, int32_t* __restrict__ fb, int* __restrict__ cnt, int r,
                                   const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                   const int32_t* __restrict__ cp, const int32_t* __restrict__ cr,
                                   int32_t* __restrict__ cell) {
    const int32_t* front = (r & 1) ? fb : fa;
    int32_t* next = (r & 1) ? fa : fb;
    const int nf = ld_vol(cnt + r % 3);
    if (blockIdx.x == 0 && threadIdx.x == 0) cnt[(r + 2) % 3] = 0;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nf; k += (int64_t)gridDim.x * blockDim.x) {
        const int u = front[k], c = ld_cg(cell + u);
        for (int dir = 0; dir < 2; dir++) {
            const int32_t* p = dir ? cp : rp;
            const int32_t* a = dir ? cr : ci;
            for (int e = p[u]; e < p[u + 1]; e++) {
                const int w = a[e];
                if (ld_cg(cell + w) != NOLAB) continue;
                if (atomicCAS(cell + w, NOLAB, c) == NOLAB) next[atomicAdd(cnt + (r + 1) % 3, 1)] = w;
            }
        }
    }
}
static __global__ void k_seed2(int32_t n, int32_t* __restrict__ cell, int32_t* __restrict__ front, int* __restrict__ cnt) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const bool s = is_seed((int)v);
        cell[v] = s ? (int)v : NOLAB;             // a cell is named by its seed
        if (s) front[atomicAdd(cnt, 1)] = (int)v;
    }
}
// cell key (seed ID >> CELL_SHIFT: nearly unique per cell, ordered like the seeds);
// vertices no seed reached form cells of their own ID range
static __global__ void k_cell_hist(int32_t n, int32_t* __restrict__ lab, int32_t* __restrict__ hist) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int c = lab[v];
        if (c == NOLAB) c = (int)v;
        c >>= CELL_SHIFT;
        lab[v] = c;
        atomicAdd(hist + c, 1);
    }
}
static __global__ void k_cell_place(int32_t n, const int32_t* __restrict__ key, const int32_t* __restrict__ start,
                                    int32_t* __restrict__ cursor, int32_t* __restrict__ pos, int32_t* __restrict__ orig) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int c = key[v];
        const int j = start[c] + atomicAdd(cursor + c, 1);
        pos[v] = j;
        orig[j] = (int)v;
    }
}
// one CTA per cell: sort the cell's storage slots by caller ID (bitonic sort in shared
// memory), so that a tile holding part of a cell holds a compact piece of it (the
// atomic placement above leaves the members in arbitrary order).  Cells larger than
// SORT_MAX keep the arbitrary order (only the pass count depends on it).
constexpr int SORT_MAX = 8192;
constexpr int SORT_THREADS = 1024;
static __global__ void __launch_bounds__(SORT_THREADS) k_cell_sort(int64_t nkeys, const int32_t* __restrict__ start,
                                                                  int32_t* __restrict__ orig, int32_t* __restrict__ pos) {
    __shared__ int32_t sk[SORT_MAX];
    for (int64_t c = blockIdx.x; c < nkeys; c += gridDim.x) {
        const int b = start[c], sz = start[c + 1] - b;
        if (sz <= 1 || sz > SORT_MAX) continue;
        int m = 1;
        while (m < sz) m <<= 1;
        for (int k = threadIdx.x; k < m; k += SORT_THREADS) sk[k] = k < sz ? orig[b + k] : 0x7FFFFFFF;
        __syncthreads();
        for (int k = 2; k <= m; k <<= 1)
            for (int j = k >> 1; j > 0; j >>= 1) {
                for (int t = threadIdx.x; t < m; t += SORT_THREADS) {
                    const int o = t ^ j;
                    if (o > t) {
                        const int x = sk[t], y = sk[o];
                        if (((t & k) == 0) == (x > y)) { sk[t] = y; sk[o] = x; }
                    }
                }
                __syncthreads();
            }
        for (int k = threadIdx.x; k < sz; k += SORT_THREADS) {
            const int v = sk[k];
            orig[b + k] = v;
            pos[v] = b + k;
        }
        __syncthreads();
    }
}
static __global__ void k_perm_deg(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ pos,
                                  int32_t* __restrict__ deg) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        deg[pos[v]] = rp[v + 1] - rp[v];
}
static __global__ void k_perm_fill(int32_t n, const int32_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                   const int32_t* __restrict__ pos, const int32_t* __restrict__ rp2,
                                   int32_t* __restrict__ ci2) {
    const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    int o = rp2[pos[v]];
    for (int e = rp[v]; e < rp[v + 1]; e++) ci2[o++] = pos[ci[e]];
}

}  // namespace reo
}  // namespace eclscc
