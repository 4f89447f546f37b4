// scan.cuh -- exclusive prefix sums (int32 and int4 lanes) for compaction offsets.
//
// Three launches: per-block totals, a single-block scan of the totals, then a re-scan of
// each block with its offset.  Used on per-vertex in-degrees (CSC build, n entries) and on
// per-warp (alive, out, in) counts of the edge-removal phase (na/32 entries).
#pragma once
#include "common.cuh"

namespace eclscc {

constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;

struct I1 {
    int x;
    __device__ __forceinline__ static I1 zero() { return {0}; }
    __device__ __forceinline__ I1 operator+(const I1& o) const { return {x + o.x}; }
    __device__ __forceinline__ I1 shfl_up(int d) const { return {__shfl_up_sync(FULL, x, d)}; }
};
struct __align__(16) I3 {
    int x, y, z, w;
    __device__ __forceinline__ static I3 zero() { return {0, 0, 0, 0}; }
    __device__ __forceinline__ I3 operator+(const I3& o) const { return {x + o.x, y + o.y, z + o.z, w + o.w}; }
    __device__ __forceinline__ I3 shfl_up(int d) const {
        return {__shfl_up_sync(FULL, x, d), __shfl_up_sync(FULL, y, d), __shfl_up_sync(FULL, z, d),
                __shfl_up_sync(FULL, w, d)};
    }
};

// block-wide exclusive scan of one value per thread; returns exclusive prefix, sets total
template <typename T>
__device__ __forceinline__ T block_excl_scan(T v, T& total) {
    __shared__ T wsum[SCAN_THREADS / WARP];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    T inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T t = inc.shfl_up(o);
        if (lane >= o) inc = inc + t;
    }
    if (lane == 31) wsum[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        T s = lane < SCAN_THREADS / WARP ? wsum[lane] : T::zero();
        T si = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            T t = si.shfl_up(o);
            if (lane >= o) si = si + t;
        }
        if (lane < SCAN_THREADS / WARP) wsum[lane] = si;  // inclusive
    }
    __syncthreads();
    T woff = wid > 0 ? wsum[wid - 1] : T::zero();
    total = wsum[SCAN_THREADS / WARP - 1];
    __syncthreads();
    T exw = inc.shfl_up(1);  // warp-exclusive prefix
    if (lane == 0) exw = T::zero();
    return woff + exw;
}

template <typename T>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_reduce(const T* __restrict__ in, int64_t N, T* __restrict__ bsum) {
    const int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
    T acc = T::zero();
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; k++)
        if (base + k < N) acc = acc + in[base + k];
    T total;
    block_excl_scan(acc, total);
    if (threadIdx.x == 0) bsum[blockIdx.x] = total;
}

// single block: exclusive scan of nb block totals in place; writes the grand total
template <typename T>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_top(T* __restrict__ bsum, int64_t nb, T* __restrict__ grand) {
    T carry = T::zero();
    for (int64_t base = 0; base < nb; base += SCAN_THREADS) {
        const int64_t i = base + threadIdx.x;
        T v = i < nb ? bsum[i] : T::zero();
        T total;
        T ex = block_excl_scan(v, total);
        if (i < nb) bsum[i] = carry + ex;
        carry = carry + total;
    }
    if (threadIdx.x == 0) *grand = carry;
}

// out[i] = exclusive prefix (N entries); if out_total_at_N, out[N] = grand total
template <typename T>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_apply(const T* __restrict__ in, int64_t N, const T* __restrict__ bsum,
                                                             T* __restrict__ out, const T* __restrict__ grand, int write_total) {
    const int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
    T vals[SCAN_ITEMS];
    T acc = T::zero();
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; k++) {
        vals[k] = (base + k < N) ? in[base + k] : T::zero();
        acc = acc + vals[k];
    }
    T total;
    T ex = block_excl_scan(acc, total) + bsum[blockIdx.x];
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; k++) {
        if (base + k < N) out[base + k] = ex;
        ex = ex + vals[k];
    }
    if (write_total && blockIdx.x == 0 && threadIdx.x == 0) out[N] = *grand;
}

// k_scan_top folded into the apply for small scans (nb <= SCAN_FOLD_NB block totals, e.g. the
// per-warp compaction counts: C4 251 blocks): every block sums the totals of the blocks before
// it itself (at most SCAN_FOLD_NB loads, L2-resident), the last block writes the grand total.
// One launch less per scan.
constexpr int64_t SCAN_FOLD_NB = 512;
template <typename T>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_apply_fold(const T* __restrict__ in, int64_t N, const T* __restrict__ bsum,
                                                                  T* __restrict__ out, T* __restrict__ grand, int write_total) {
    __shared__ T s_part[SCAN_THREADS / WARP];
    T c = T::zero();
    for (int64_t b = threadIdx.x; b < blockIdx.x; b += SCAN_THREADS) c = c + bsum[b];
    // block sum of the partial carries (warp shuffles, then one warp)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        T t = c.shfl_up(o);        // (shfl_up then add from the top lane: inclusive scan; lane 31 holds the sum)
        if ((threadIdx.x & 31) >= o) c = c + t;
    }
    if ((threadIdx.x & 31) == 31) s_part[threadIdx.x >> 5] = c;
    __syncthreads();
    T carry = T::zero();
#pragma unroll
    for (int w = 0; w < SCAN_THREADS / WARP; w++) carry = carry + s_part[w];
    __syncthreads();
    const int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
    T vals[SCAN_ITEMS];
    T acc = T::zero();
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; k++) {
        vals[k] = (base + k < N) ? in[base + k] : T::zero();
        acc = acc + vals[k];
    }
    T total;
    T ex = block_excl_scan(acc, total) + carry;
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; k++) {
        if (base + k < N) out[base + k] = ex;
        ex = ex + vals[k];
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
        const T g = carry + total;
        *grand = g;
        if (write_total) out[N] = g;
    }
}

}  // namespace eclscc
