// Exclusive prefix sums (reduce-then-scan, 3 launches).  Used by the frontier
// allocator (offsets of the next level, Algorithm 2 line 30
// "offsets <- CUBSCAN(counts)") and by preprocessing.
#include "common.cuh"

namespace mce {

namespace {
constexpr int kThreads = 256;
constexpr int kItems = 16;
constexpr int kTile = kThreads * kItems;

__device__ __forceinline__ int64_t block_exclusive_sum(int64_t x, int64_t *total) {
    __shared__ int64_t warp_sums[kThreads / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int64_t v = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int64_t y = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += y;
    }
    if (lane == 31) warp_sums[warp] = v;
    __syncthreads();
    if (warp == 0) {
        int64_t w = lane < kThreads / 32 ? warp_sums[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int64_t y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        if (lane < kThreads / 32) warp_sums[lane] = w;
    }
    __syncthreads();
    int64_t warp_prefix = warp ? warp_sums[warp - 1] : 0;
    *total = warp_sums[kThreads / 32 - 1];
    __syncthreads();
    return warp_prefix + v - x;
}

template <typename T>
__global__ void __launch_bounds__(kThreads) tile_reduce(const T *__restrict__ in, int64_t n, int64_t *partial) {
    int64_t base = (int64_t)blockIdx.x * kTile + (int64_t)threadIdx.x * kItems;
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i)
        if (base + i < n) s += (int64_t)in[base + i];
    int64_t total;
    block_exclusive_sum(s, &total);
    if (threadIdx.x == 0) partial[blockIdx.x] = total;
}

// single block: exclusive scan of partial[0..tiles) in place, partial[tiles] = total
__global__ void __launch_bounds__(kThreads) scan_partials(int64_t *partial, int64_t tiles) {
    int64_t carry = 0;
    for (int64_t b0 = 0; b0 < tiles; b0 += kThreads) {
        int64_t i = b0 + threadIdx.x;
        int64_t x = i < tiles ? partial[i] : 0;
        int64_t total;
        int64_t ex = block_exclusive_sum(x, &total);
        if (i < tiles) partial[i] = carry + ex;
        carry += total;
    }
    if (threadIdx.x == 0) partial[tiles] = carry;
}

template <typename T>
__global__ void __launch_bounds__(kThreads) tile_scan(const T *__restrict__ in, int64_t *__restrict__ out, int64_t n,
                                                      const int64_t *__restrict__ partial, int64_t tiles) {
    int64_t base = (int64_t)blockIdx.x * kTile + (int64_t)threadIdx.x * kItems;
    int64_t v[kItems];
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        v[i] = base + i < n ? (int64_t)in[base + i] : 0;
        s += v[i];
    }
    int64_t total;
    int64_t run = block_exclusive_sum(s, &total) + partial[blockIdx.x];
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        if (base + i < n) out[base + i] = run;
        run += v[i];
    }
    if (blockIdx.x == tiles - 1 && threadIdx.x == 0) out[n] = partial[tiles];
}

template <typename T>
void exclusive_scan(const T *in, int64_t *out, int64_t n, int64_t *tmp, cudaStream_t s) {
    if (n <= 0) {
        MCE_CUDA(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
        return;
    }
    int64_t tiles = ceil_div(n, kTile);
    tile_reduce<T><<<(unsigned)tiles, kThreads, 0, s>>>(in, n, tmp);
    MCE_LAUNCH_CHECK();
    scan_partials<<<1, kThreads, 0, s>>>(tmp, tiles);
    MCE_LAUNCH_CHECK();
    tile_scan<T><<<(unsigned)tiles, kThreads, 0, s>>>(in, out, n, tmp, tiles);
    MCE_LAUNCH_CHECK();
}
}  // namespace

int64_t scan_tmp_items(int64_t n) { return ceil_div(n > 0 ? n : 1, kTile) + 1; }

void exclusive_scan_i32(const int32_t *in, int64_t *out, int64_t n, int64_t *tmp, cudaStream_t s) {
    exclusive_scan<int32_t>(in, out, n, tmp, s);
}
void exclusive_scan_i64(const int64_t *in, int64_t *out, int64_t n, int64_t *tmp, cudaStream_t s) {
    exclusive_scan<int64_t>(in, out, n, tmp, s);
}

}  // namespace mce
