// Shared host/device helpers of libmce_b200 (NOT shared with oracle/).
#pragma once

#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <stdexcept>
#include <string>
#include <vector>

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
// per-device caching allocator (alloc.cu): freed blocks are kept and handed
// out again, so a new graph handle, a new phase or a regrown buffer does not
// pay cudaMalloc/cudaFree (cudaFree serialises the whole device).  Sizes are
// rounded (4 KiB below 1 MiB, 2 MiB above); a cached block is reused for a
// request of at least 3/4 of its size.  mce_empty_cache() returns it all.
// ---------------------------------------------------------------------------
void *dev_alloc(size_t bytes);           // throws MCE_ERR_NOMEM / MCE_ERR_CUDA
void dev_free(void *p, size_t bytes);    // bytes = the size passed to dev_alloc
size_t dev_cached_bytes();               // free bytes held by the cache on this device
size_t dev_free_memory();                // cudaMemGetInfo free bytes, re-queried at most once a second
void dev_empty_cache();
void *host_pinned(size_t bytes, int slot = 0);  // per-device pinned staging (grow-only; slot per thread role)

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
        if (count) p = static_cast<T *>(dev_alloc(sizeof(T) * count));
        n = count;
    }
    // keep the current allocation when it is large enough (no cudaMalloc/cudaFree)
    void ensure(size_t count) {
        if (n < count || !p) alloc(count);
    }
    void release() {
        if (p) dev_free(p, sizeof(T) * n);
        p = nullptr;
        n = 0;
    }
    T *get() const { return p; }
    size_t bytes() const { return sizeof(T) * n; }
};

// pinned host staging (small scalar read-backs without pageable copies);
// the memory is the device's shared staging block (host_pinned)
struct PinnedBuf {
    int slot = 0;
    template <typename T>
    T *get(size_t count) {
        return reinterpret_cast<T *>(host_pinned(count * sizeof(T), slot));
    }
};

// host<->device round trips are the fixed cost of every level; they are
// counted (per thread) so the bench can report them
extern thread_local int64_t g_syncs;
inline void stream_sync(cudaStream_t s) {
    ++g_syncs;
    MCE_CUDA(cudaStreamSynchronize(s));
}

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ---------------------------------------------------------------------------
// grow-only device scratch pool, stream-ordered: take() bumps a pointer,
// reset() releases everything taken since the last reset.  A request that
// does not fit spills to its own cudaMalloc; the next reset() frees the
// spills and regrows the main block to the high-water mark, so from the
// second call on a phase runs without any cudaMalloc/cudaFree (both of which
// serialise the device).
// ---------------------------------------------------------------------------
class Pool {
   public:
    Pool() = default;
    Pool(const Pool &) = delete;
    Pool &operator=(const Pool &) = delete;
    ~Pool() {
        for (auto &q : spill_) dev_free(q.first, q.second);
    }
    template <typename T>
    T *take(int64_t count) {
        const size_t bytes = ((size_t)(count > 0 ? count : 1) * sizeof(T) + 255) / 256 * 256;
        if (top_ + bytes <= main_.n) {
            T *q = reinterpret_cast<T *>(main_.p + top_);
            top_ += bytes;
            return q;
        }
        void *q = dev_alloc(bytes);
        spill_.push_back({q, bytes});
        spill_bytes_ += bytes;
        return reinterpret_cast<T *>(q);
    }
    void reset() {
        if (!spill_.empty()) {
            const size_t want = top_ + spill_bytes_;
            for (auto &q : spill_) dev_free(q.first, q.second);
            spill_.clear();
            spill_bytes_ = 0;
            if (want > main_.n) main_.alloc(want + want / 4);
        }
        top_ = 0;
    }
    size_t capacity() const { return main_.n; }

   private:
    DevBuf<uint8_t> main_;
    size_t top_ = 0;
    std::vector<std::pair<void *, size_t>> spill_;
    size_t spill_bytes_ = 0;
};

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
