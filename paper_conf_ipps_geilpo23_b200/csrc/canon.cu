// Canonical read-out of the stored maximum cliques on the device (DESIGN.md
// §8 row a9, reading 1): every clique's vertices ascending, the list in
// lexicographic order.  Rows arrive in search order (root first, then the
// vertices along the Fig. 1 parent chain), so
//   1. each row is sorted by one block (bitonic network in shared memory);
//   2. the row indices are ordered by a CUB merge sort (library primitive)
//      with a lexicographic row comparator: O(n log n) comparisons that stop
//      at the first differing column, instead of one radix pass per column
//      pair (R-MAT's 223-vertex cliques took 112 passes);
//   3. the rows are gathered in that order.
// The host receives one contiguous block instead of sorting 10^5+ long rows.
#include <cub/device/device_merge_sort.cuh>

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

struct RowLess {
    const int32_t *rows;
    int width;
    __device__ __forceinline__ bool operator()(const int32_t &a, const int32_t &b) const {
        const int32_t *x = rows + (int64_t)a * width, *y = rows + (int64_t)b * width;
        for (int c = 0; c < width; ++c) {
            const int32_t u = __ldg(x + c), v = __ldg(y + c);
            if (u != v) return u < v;
        }
        return false;
    }
};

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
    int32_t *perm = pool.take<int32_t>(nrows);
    iota_i32<<<grid_for(nrows, 256), 256, 0, s>>>(nrows, perm);
    MCE_LAUNCH_CHECK();
    if (nrows > 1) {
        (void)n_vertices;
        size_t tmp_bytes = 0;
        const RowLess less{rows, width};
        MCE_CUDA(cub::DeviceMergeSort::SortKeys(nullptr, tmp_bytes, perm, (int64_t)nrows, less, s));
        void *tmp = pool.take<uint8_t>((int64_t)tmp_bytes);
        MCE_CUDA(cub::DeviceMergeSort::SortKeys(tmp, tmp_bytes, perm, (int64_t)nrows, less, s));
    }
    gather_rows<<<grid_for(nrows * width, 256), 256, 0, s>>>(rows, nrows, width, perm, out);
    MCE_LAUNCH_CHECK();
    return true;
}

}  // namespace mce
