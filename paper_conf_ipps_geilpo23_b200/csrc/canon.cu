// Canonical read-out of the stored maximum cliques on the device (DESIGN.md
// §8 row a9, reading 1): every clique's vertices ascending, the list in
// lexicographic order.  Rows arrive in search order (root first, then the
// vertices along the Fig. 1 parent chain), so
//   1. each row is sorted by one block (bitonic network in shared memory);
//   2. the rows are ordered by an LSD radix sort over the columns, two
//      columns per stable 64-bit CUB radix pass (library primitive), from the
//      last column pair to the first;
//   3. the rows are gathered in that order.
// The host receives one contiguous block instead of sorting 10^5+ long rows.
#include <cub/device/device_radix_sort.cuh>

#include "canon.cuh"

namespace mce {

namespace {

constexpr int kSortThreads = 256;

__global__ void __launch_bounds__(kSortThreads) sort_each_row(int32_t *rows, int64_t nrows, int width, int p2) {
    extern __shared__ int32_t buf[];
    for (int64_t r = blockIdx.x; r < nrows; r += gridDim.x) {
        int32_t *row = rows + r * width;
        for (int i = threadIdx.x; i < p2; i += blockDim.x) buf[i] = i < width ? row[i] : INT32_MAX;
        __syncthreads();
        for (int size = 2; size <= p2; size <<= 1) {
            for (int stride = size >> 1; stride > 0; stride >>= 1) {
                for (int i = threadIdx.x; i < p2; i += blockDim.x) {
                    const int j = i ^ stride;
                    if (j > i) {
                        const bool up = (i & size) == 0;
                        const int32_t a = buf[i], b = buf[j];
                        if ((a > b) == up) {
                            buf[i] = b;
                            buf[j] = a;
                        }
                    }
                }
                __syncthreads();
            }
        }
        for (int i = threadIdx.x; i < width; i += blockDim.x) row[i] = buf[i];
        __syncthreads();
    }
}

__global__ void iota_i32(int64_t n, int32_t *out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (int32_t)i;
}

// key of row perm[i] for columns (c0, c1): value(c0) in the high word
__global__ void column_keys(const int32_t *__restrict__ rows, int64_t nrows, int width, int c0, int c1,
                            const int32_t *__restrict__ perm, uint64_t *keys) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrows; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t *row = rows + (int64_t)perm[i] * width;
        const uint64_t hi = c0 >= 0 ? (uint32_t)row[c0] : 0u;
        keys[i] = (hi << 32) | (uint32_t)row[c1];
    }
}

__global__ void gather_rows(const int32_t *__restrict__ rows, int64_t nrows, int width,
                            const int32_t *__restrict__ perm, int32_t *out) {
    const int64_t total = nrows * width;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = t / width, c = t - i * width;
        out[t] = rows[(int64_t)perm[i] * width + c];
    }
}

}  // namespace

bool canonicalize_device(int32_t *rows, int64_t nrows, int width, int64_t n_vertices, int32_t *out, Pool &pool,
                         cudaStream_t s) {
    if (nrows <= 0 || width <= 0) return true;
    int p2 = 1;
    while (p2 < width) p2 <<= 1;
    if (p2 > 8192) return false;  // rows wider than shared memory: the host sorts them
    sort_each_row<<<grid_for(nrows, 1, 16), kSortThreads, sizeof(int32_t) * p2, s>>>(rows, nrows, width, p2);
    MCE_LAUNCH_CHECK();
    int32_t *perm = pool.take<int32_t>(nrows), *perm2 = pool.take<int32_t>(nrows);
    uint64_t *keys = pool.take<uint64_t>(nrows), *keys2 = pool.take<uint64_t>(nrows);
    iota_i32<<<grid_for(nrows, 256), 256, 0, s>>>(nrows, perm);
    MCE_LAUNCH_CHECK();
    if (nrows > 1) {
        int vbits = 1;
        while (vbits < 31 && (1ll << vbits) < n_vertices) ++vbits;
        size_t tmp_bytes = 0;
        MCE_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, keys, keys2, perm, perm2, (int)nrows, 0, 64, s));
        void *tmp = pool.take<uint8_t>((int64_t)tmp_bytes);
        // LSD over column pairs (c0, c1), last pair first; stable passes
        for (int c1 = width - 1; c1 >= 0; c1 -= 2) {
            const int c0 = c1 - 1;
            column_keys<<<grid_for(nrows, 256), 256, 0, s>>>(rows, nrows, width, c0, c1, perm, keys);
            MCE_LAUNCH_CHECK();
            const int end_bit = c0 >= 0 ? 32 + vbits : vbits;
            MCE_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, keys, keys2, perm, perm2, (int)nrows, 0, end_bit,
                                                     s));
            std::swap(perm, perm2);
        }
    }
    gather_rows<<<grid_for(nrows * width, 256), 256, 0, s>>>(rows, nrows, width, perm, out);
    MCE_LAUNCH_CHECK();
    return true;
}

}  // namespace mce
