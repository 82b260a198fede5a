// Shared host/device helpers of libmce_b200 (NOT shared with oracle/).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <stdexcept>
#include <string>

namespace mce {

// ---------------------------------------------------------------------------
// errors: C++ exceptions inside the library, mce_status at the C boundary
// ---------------------------------------------------------------------------
struct Error : std::runtime_error {
    int status;
    Error(int s, const std::string &m) : std::runtime_error(m), status(s) {}
};

[[noreturn]] void fail(int status, const std::string &msg);

#define MCE_CUDA(call)                                                                                  \
    do {                                                                                                \
        cudaError_t _e = (call);                                                                        \
        if (_e != cudaSuccess) {                                                                        \
            ::mce::fail(_e == cudaErrorMemoryAllocation ? 3 : 2,                                        \
                        std::string(#call) + ": " + cudaGetErrorString(_e) + " @ " + __FILE__ + ":" +   \
                            std::to_string(__LINE__));                                                  \
        }                                                                                               \
    } while (0)

#define MCE_LAUNCH_CHECK() MCE_CUDA(cudaGetLastError())

// ---------------------------------------------------------------------------
// owning device buffer
// ---------------------------------------------------------------------------
template <typename T>
struct DevBuf {
    T *p = nullptr;
    size_t n = 0;
    DevBuf() = default;
    explicit DevBuf(size_t count) { alloc(count); }
    DevBuf(const DevBuf &) = delete;
    DevBuf &operator=(const DevBuf &) = delete;
    DevBuf(DevBuf &&o) noexcept : p(o.p), n(o.n) { o.p = nullptr; o.n = 0; }
    DevBuf &operator=(DevBuf &&o) noexcept {
        if (this != &o) { release(); p = o.p; n = o.n; o.p = nullptr; o.n = 0; }
        return *this;
    }
    ~DevBuf() { release(); }
    void alloc(size_t count) {
        release();
        n = count;
        if (count) MCE_CUDA(cudaMalloc(&p, sizeof(T) * count));
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
    T *get() const { return p; }
    size_t bytes() const { return sizeof(T) * n; }
};

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// grid size for a grid-stride kernel: a multiple of the SM count
int grid_for(int64_t work_items, int threads_per_block, int max_blocks_per_sm = 8);
int num_sms();

// ---------------------------------------------------------------------------
// device helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// first index in sorted a[lo, hi) with a[i] >= key
__device__ __forceinline__ int64_t lower_bound_i32(const int32_t *__restrict__ a, int64_t lo, int64_t hi,
                                                   int32_t key) {
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (__ldg(a + mid) < key)
            lo = mid + 1;
        else
            hi = mid;
    }
    return lo;
}

__device__ __forceinline__ bool contains_sorted(const int32_t *__restrict__ a, int64_t lo, int64_t hi,
                                                int32_t key) {
    int64_t p = lower_bound_i32(a, lo, hi, key);
    return p < hi && __ldg(a + p) == key;
}

// ---------------------------------------------------------------------------
// scan primitives (scan.cu)
// ---------------------------------------------------------------------------
// out[0..n] = exclusive prefix sums of in[0..n-1]; out[n] = total.  in may be int32 or int64.
void exclusive_scan_i32(const int32_t *in, int64_t *out, int64_t n, int64_t *tmp, cudaStream_t s);
void exclusive_scan_i64(const int64_t *in, int64_t *out, int64_t n, int64_t *tmp, cudaStream_t s);
// bytes of int64 scratch the scans need for n items
int64_t scan_tmp_items(int64_t n);

}  // namespace mce
