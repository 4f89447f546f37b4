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
#include <cub/block/block_radix_sort.cuh>

#include "common.cuh"

namespace eclscc {
namespace reo {

constexpr int CELL_SHIFT = 11;        // ~2048 vertices per cell
constexpr int NOLAB = 0x7FFFFFFF;
constexpr int BFS_STAGE = 4096;       // claimed vertices staged per block and level

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
    const int lane = threadIdx.x & 31;
    // whole warps iterate (ballots below); claimed vertices are staged in shared memory and
    // appended with ONE global atomic per block at the end (per-warp atomics on the single
    // frontier counter serialised in L2); a full stage spills with per-warp atomics
    __shared__ int s_buf[BFS_STAGE];
    __shared__ int s_n, s_base;
    if (threadIdx.x == 0) s_n = 0;
    __syncthreads();
    int* gcnt = cnt + (r + 1) % 3;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t k0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x - lane; k0 < nf; k0 += stride) {
        const int64_t k = k0 + lane;
        const bool act = k < nf;
        int u = 0, c = 0, b0 = 0, e0 = 0, b1 = 0, e1 = 0;
        if (act) {
            u = front[k];
            c = ld_cg(cell + u);
            b0 = rp[u]; e0 = rp[u + 1]; b1 = cp[u]; e1 = cp[u + 1];
        }
        int n0 = e0 - b0, n1 = e1 - b1;
        for (int j0 = 0;; j0 += 4) {                   // neighbours j0..j0+3 of every lane's vertex
            if (!__any_sync(FULL, j0 < n0 + n1)) break;
            // the adjacency loads, then the cell loads, of a batch are issued before use
            int w[4], cw[4];
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int j = j0 + q;
                w[q] = j < n0 + n1 ? (j < n0 ? ci[b0 + j] : cr[b1 + j - n0]) : -1;
            }
#pragma unroll
            for (int q = 0; q < 4; q++) cw[q] = w[q] >= 0 ? ld_cg(cell + w[q]) : 0;
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const bool got = w[q] >= 0 && cw[q] == NOLAB && atomicCAS(cell + w[q], NOLAB, c) == NOLAB;
                const unsigned m = __ballot_sync(FULL, got);
                if (m) {
                    int at = 0;
                    if (lane == __ffs(m) - 1) at = atomicAdd(&s_n, __popc(m));
                    at = __shfl_sync(FULL, at, __ffs(m) - 1);
                    const int slot = at + __popc(m & ((1u << lane) - 1));
                    if (got && slot < BFS_STAGE) s_buf[slot] = w[q];
                    const unsigned sp = __ballot_sync(FULL, got && slot >= BFS_STAGE);
                    if (sp) {                                   // stage full: straight to the frontier
                        int g0 = 0;
                        if (lane == __ffs(sp) - 1) g0 = atomicAdd(gcnt, __popc(sp));
                        g0 = __shfl_sync(FULL, g0, __ffs(sp) - 1);
                        if (got && slot >= BFS_STAGE) next[g0 + __popc(sp & ((1u << lane) - 1))] = w[q];
                    }
                }
            }
        }
    }
    __syncthreads();
    const int ns = min(s_n, BFS_STAGE);
    if (threadIdx.x == 0) s_base = ns ? atomicAdd(gcnt, ns) : 0;
    __syncthreads();
    for (int i = threadIdx.x; i < ns; i += blockDim.x) next[s_base + i] = s_buf[i];
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
// lanes with equal keys (consecutive vertices mostly share a cell) add once per group
static __global__ void k_cell_hist_agg(int32_t n, int32_t* __restrict__ lab, int32_t* __restrict__ hist) {
    const int lane = threadIdx.x & 31;
    for (int64_t v0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x - lane; v0 < n; v0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = v0 + lane;
        int c = -1;
        if (v < n) {
            c = lab[v];
            if (c == NOLAB) c = (int)v;
            c >>= CELL_SHIFT;
            lab[v] = c;
        }
        const unsigned grp = __match_any_sync(FULL, c);
        if (c >= 0 && lane == __ffs(grp) - 1) atomicAdd(hist + c, __popc(grp));
    }
}
static __global__ void k_cell_place(int32_t n, const int32_t* __restrict__ key, const int32_t* __restrict__ start,
                                    int32_t* __restrict__ cursor, int32_t* __restrict__ pos, int32_t* __restrict__ orig) {
    const int lane = threadIdx.x & 31;
    for (int64_t v0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x - lane; v0 < n; v0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = v0 + lane;
        const int c = v < n ? key[v] : -1;
        const unsigned grp = __match_any_sync(FULL, c);       // one atomic per key group
        const int leader = __ffs(grp) - 1;
        int at = 0;
        if (c >= 0 && lane == leader) at = atomicAdd(cursor + c, __popc(grp));
        at = __shfl_sync(FULL, at, leader);
        if (c >= 0) {
            const int j = start[c] + at + __popc(grp & ((1u << lane) - 1));
            pos[v] = j;
            orig[j] = (int)v;
        }
    }
}
// one CTA per cell: sort the cell's storage slots by caller ID (radix sort in shared
// memory, below), so that a tile holding part of a cell holds a compact piece of it (the
// atomic placement above leaves the members in arbitrary order).  Cells larger than
// SORT_MAX keep the arbitrary order (only the pass count depends on it).
constexpr int SORT_MAX = 8192;
constexpr int SORT_THREADS = 256;
// A cell's members (caller IDs, all < 2^bits) sorted in shared memory by a block radix sort
// (the CUB building block inside this kernel; round 1 used a bitonic network: 78 barrier
// stages per 4096-member cell, C4 lex 1.48 ms for the kernel), in two sizes: cells up to
// 4096 and up to SORT_MAX members.  Loads are striped (the sort ignores the input order),
// results come back striped (coalesced stores).
template <int ITEMS>
using CellSort = cub::BlockRadixSort<unsigned, SORT_THREADS, ITEMS>;
template <int ITEMS>
__device__ __forceinline__ void sort_cell(int32_t* __restrict__ orig, int32_t* __restrict__ pos, int b, int sz, int bits,
                                          typename CellSort<ITEMS>::TempStorage& tmp) {
    const unsigned pad = bits >= 32 ? 0xFFFFFFFFu : (1u << bits) - 1u;   // above every ID
    unsigned key[ITEMS];
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
        const int k = i * SORT_THREADS + threadIdx.x;
        key[i] = k < sz ? (unsigned)orig[b + k] : pad;
    }
    CellSort<ITEMS>(tmp).SortBlockedToStriped(key, 0, bits);
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
        const int k = i * SORT_THREADS + threadIdx.x;
        if (k < sz) {
            orig[b + k] = (int32_t)key[i];
            pos[key[i]] = b + k;
        }
    }
}
static __global__ void __launch_bounds__(SORT_THREADS) k_cell_sort(int64_t nkeys, const int32_t* __restrict__ start,
                                                                  int32_t* __restrict__ orig, int32_t* __restrict__ pos,
                                                                  int bits) {
    __shared__ union {
        typename CellSort<SORT_MAX / 2 / SORT_THREADS>::TempStorage small;
        typename CellSort<SORT_MAX / SORT_THREADS>::TempStorage large;
    } tmp;
    for (int64_t c = blockIdx.x; c < nkeys; c += gridDim.x) {
        const int b = start[c], sz = start[c + 1] - b;
        if (sz <= 1 || sz > SORT_MAX) continue;        // (larger cells keep the placement order)
        if (sz <= SORT_MAX / 2) sort_cell<SORT_MAX / 2 / SORT_THREADS>(orig, pos, b, sz, bits, tmp.small);
        else sort_cell<SORT_MAX / SORT_THREADS>(orig, pos, b, sz, bits, tmp.large);
        __syncthreads();                               // tmp is reused by the next cell
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
