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
// When the stored cliques use at most kMaxKeyBits distinct vertices (R-MAT:
// 223-cliques over ~250 vertices) a faster exact route is taken: every row
// becomes a bit key over the ranks of those vertices, most significant bit =
// smallest vertex.  For two sets of equal size the lexicographic order of
// their sorted lists is decided by the smallest vertex of their symmetric
// difference (the list holding it is smaller), i.e. by the key compared as a
// big integer, descending: a few stable 64-bit radix passes, and the sorted
// rows are read back from the key bits.
// The host receives one contiguous block instead of sorting 10^5+ long rows.
#include <cub/device/device_merge_sort.cuh>
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

constexpr int kMaxKeyBits = 1024;

__global__ void mark_vertices(const int32_t *__restrict__ rows, int64_t total, uint32_t *bits) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = rows[t];
        atomicOr(bits + (v >> 5), 1u << (v & 31));
    }
}

__global__ void word_popc(const uint32_t *__restrict__ bits, int64_t nw, int32_t *cnt) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (int64_t)gridDim.x * blockDim.x)
        cnt[w] = __popc(bits[w]);
}

// rank -> vertex of the marked vertices
__global__ void list_vertices(const uint32_t *__restrict__ bits, const int64_t *__restrict__ pre, int64_t nw,
                              int32_t *ulist) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (int64_t)gridDim.x * blockDim.x) {
        uint32_t b = bits[w];
        int64_t r = pre[w];
        while (b) {
            const int i = __ffs(b) - 1;
            b &= b - 1;
            ulist[r++] = (int32_t)(w * 32 + i);
        }
    }
}

// key word j of row i (KW words, word 0 most significant): bit 63 - (rank % 64) of word rank / 64
__global__ void build_keys(const int32_t *__restrict__ rows, int64_t nrows, int width,
                           const uint32_t *__restrict__ bits, const int64_t *__restrict__ pre, int KW,
                           unsigned long long *keys) {
    const int64_t total = nrows * width;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = t / width;
        const int32_t v = rows[t];
        const int64_t r = pre[v >> 5] + __popc(bits[v >> 5] & ((1u << (v & 31)) - 1u));
        atomicOr(keys + i * KW + (r >> 6), 1ull << (63 - (r & 63)));
    }
}

__global__ void key_column(const unsigned long long *__restrict__ keys, int64_t nrows, int KW, int j,
                           const int32_t *__restrict__ perm, unsigned long long *col) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrows; i += (int64_t)gridDim.x * blockDim.x)
        col[i] = keys[(int64_t)perm[i] * KW + j];
}

// row i of the output = the set bits of key perm[i], most significant first
__global__ void rows_from_keys(const unsigned long long *__restrict__ keys, int64_t nrows, int KW, int width,
                               const int32_t *__restrict__ perm, const int32_t *__restrict__ ulist, int32_t *out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrows; i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long *k = keys + (int64_t)perm[i] * KW;
        int32_t *o = out + i * width;
        int c = 0;
        for (int j = 0; j < KW && c < width; ++j) {
            unsigned long long x = k[j];
            while (x && c < width) {
                const int b = 63 - __clzll((long long)x);
                x &= ~(1ull << b);
                o[c++] = ulist[j * 64 + (63 - b)];
            }
        }
    }
}

// the bit-key route; false when the cliques use more than kMaxKeyBits vertices
bool canonicalize_by_keys(const int32_t *rows, int64_t nrows, int width, int64_t n_vertices, int32_t *out,
                          Pool &pool, cudaStream_t s) {
    const int64_t nw = (n_vertices + 31) / 32;
    uint32_t *bits = pool.take<uint32_t>(nw);
    int32_t *cnt = pool.take<int32_t>(nw);
    int64_t *pre = pool.take<int64_t>(nw + 1);
    int64_t *tmp = pool.take<int64_t>(scan_tmp_items(nw));
    MCE_CUDA(cudaMemsetAsync(bits, 0, sizeof(uint32_t) * nw, s));
    mark_vertices<<<grid_for(nrows * width, 256), 256, 0, s>>>(rows, nrows * width, bits);
    word_popc<<<grid_for(nw, 256), 256, 0, s>>>(bits, nw, cnt);
    MCE_LAUNCH_CHECK();
    exclusive_scan_i32(cnt, pre, nw, tmp, s);
    int64_t *hu = static_cast<int64_t *>(host_pinned(sizeof(int64_t)));
    MCE_CUDA(cudaMemcpyAsync(hu, pre + nw, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    MCE_CUDA(cudaStreamSynchronize(s));
    const int64_t U = *hu;
    if (U > kMaxKeyBits) return false;
    const int KW = (int)((U + 63) / 64);
    int32_t *ulist = pool.take<int32_t>(std::max<int64_t>(U, 1));
    list_vertices<<<grid_for(nw, 256), 256, 0, s>>>(bits, pre, nw, ulist);
    unsigned long long *keys = pool.take<unsigned long long>(nrows * KW);
    MCE_CUDA(cudaMemsetAsync(keys, 0, sizeof(unsigned long long) * nrows * KW, s));
    build_keys<<<grid_for(nrows * width, 256), 256, 0, s>>>(rows, nrows, width, bits, pre, KW, keys);
    MCE_LAUNCH_CHECK();
    int32_t *perm = pool.take<int32_t>(nrows), *perm2 = pool.take<int32_t>(nrows);
    unsigned long long *col = pool.take<unsigned long long>(nrows), *col2 = pool.take<unsigned long long>(nrows);
    iota_i32<<<grid_for(nrows, 256), 256, 0, s>>>(nrows, perm);
    MCE_LAUNCH_CHECK();
    size_t tb = 0;
    MCE_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, col, col2, perm, perm2, (int)nrows, 0, 64, s));
    void *tmpb = pool.take<uint8_t>((int64_t)tb);
    for (int j = KW - 1; j >= 0; --j) {  // LSD: least significant key word first, stable passes
        key_column<<<grid_for(nrows, 256), 256, 0, s>>>(keys, nrows, KW, j, perm, col);
        MCE_LAUNCH_CHECK();
        MCE_CUDA(cub::DeviceRadixSort::SortPairsDescending(tmpb, tb, col, col2, perm, perm2, (int)nrows, 0, 64, s));
        std::swap(perm, perm2);
    }
    rows_from_keys<<<grid_for(nrows, 256), 256, 0, s>>>(keys, nrows, KW, width, perm, ulist, out);
    MCE_LAUNCH_CHECK();
    return true;
}

}  // namespace

bool canonicalize_device(int32_t *rows, int64_t nrows, int width, int64_t n_vertices, int32_t *out, Pool &pool,
                         cudaStream_t s) {
    if (nrows <= 0 || width <= 0) return true;
    if (nrows > 1 && n_vertices > 0 && canonicalize_by_keys(rows, nrows, width, n_vertices, out, pool, s)) return true;
    int p2 = 1;
    while (p2 < width) p2 <<= 1;
    if (p2 > 8192) return false;  // rows wider than shared memory: the host sorts them
    sort_each_row<<<grid_for(nrows, 1, 16), kSortThreads, sizeof(int32_t) * p2, s>>>(rows, nrows, width, p2);
    MCE_LAUNCH_CHECK();
    int32_t *perm = pool.take<int32_t>(nrows);
    iota_i32<<<grid_for(nrows, 256), 256, 0, s>>>(nrows, perm);
    MCE_LAUNCH_CHECK();
    if (nrows > 1) {
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
