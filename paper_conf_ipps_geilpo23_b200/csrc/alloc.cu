// Per-device caching allocator and pinned staging (see common.cuh).
//
// Safety: a block is handed back to the cache only when no kernel can still
// touch it.  Every public call of the library synchronises its stream before
// returning, and the internal frees (Pool::reset at the start of a phase, a
// workspace regrow) happen after such a synchronisation, so a cached block is
// never reused while in flight, whichever stream the next user runs on.
#include <chrono>
#include <map>
#include <mutex>
#include <unordered_map>

#include "common.cuh"
#include "mce.h"

namespace mce {

thread_local int64_t g_syncs = 0;

namespace {

struct DeviceCache {
    std::multimap<size_t, void *> free_blocks;  // rounded size -> block
    size_t cached = 0;
    size_t free_mem = 0;                        // last cudaMemGetInfo answer
    std::chrono::steady_clock::time_point free_at;
    void *pinned[2] = {nullptr, nullptr};  // slot 0: the calling thread, slot 1: the overlapped heuristic
    size_t pinned_bytes[2] = {0, 0};
};

std::mutex g_mu;
std::unordered_map<int, DeviceCache> g_cache;

int current_device() {
    int d = 0;
    MCE_CUDA(cudaGetDevice(&d));
    return d;
}

size_t round_size(size_t bytes) {
    if (bytes <= (1u << 20)) return (bytes + 4095) / 4096 * 4096;
    return (bytes + (2u << 20) - 1) / (2u << 20) * (2u << 20);
}

void release_all(DeviceCache &c) {
    for (auto &b : c.free_blocks) cudaFree(b.second);
    c.free_blocks.clear();
    c.cached = 0;
}

}  // namespace

void *dev_alloc(size_t bytes) {
    const size_t r = round_size(bytes);
    const int dev = current_device();
    {
        std::lock_guard<std::mutex> lk(g_mu);
        DeviceCache &c = g_cache[dev];
        auto it = c.free_blocks.lower_bound(r);
        // reuse a block of at most 4/3 of the request.  The caller frees with its
        // own size, so the block may come back under a smaller key than its real
        // size: always safe (it is only ever handed out for smaller requests).
        if (it != c.free_blocks.end() && it->first - it->first / 4 <= r) {
            void *p = it->second;
            c.cached -= it->first;
            c.free_blocks.erase(it);
            return p;
        }
    }
    void *p = nullptr;
    cudaError_t e = cudaMalloc(&p, r);
    if (e == cudaErrorMemoryAllocation) {  // drop the cache and retry once
        cudaGetLastError();
        dev_empty_cache();
        e = cudaMalloc(&p, r);
    }
    if (e != cudaSuccess) {
        cudaGetLastError();
        fail(e == cudaErrorMemoryAllocation ? MCE_ERR_NOMEM : MCE_ERR_CUDA,
             std::string("cudaMalloc(") + std::to_string(r) + "): " + cudaGetErrorString(e));
    }
    return p;
}

// The cache keeps at most a quarter of the device's memory: blocks beyond it
// go back to the driver at once, so a run that needed a huge frontier does not
// leave the device full for the rest of the process (other allocators --
// PyTorch's -- cannot see or reclaim what this cache holds).
static size_t cache_cap(int dev) {
    static size_t cap[64] = {0};
    if (dev >= 0 && dev < 64 && !cap[dev]) {
        size_t f = 0, t = 0;
        if (cudaMemGetInfo(&f, &t) == cudaSuccess) cap[dev] = t / 4;
    }
    return dev >= 0 && dev < 64 && cap[dev] ? cap[dev] : (size_t)16 << 30;
}

void dev_free(void *p, size_t bytes) {
    if (!p) return;
    const size_t r = round_size(bytes);
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return;
    const size_t cap = cache_cap(dev);
    std::lock_guard<std::mutex> lk(g_mu);
    DeviceCache &c = g_cache[dev];
    if (c.cached + r > cap) {
        cudaFree(p);
        return;
    }
    c.free_blocks.emplace(r, p);
    c.cached += r;
}

size_t dev_cached_bytes() {
    const int dev = current_device();
    std::lock_guard<std::mutex> lk(g_mu);
    return g_cache[dev].cached;
}

void dev_empty_cache() {
    const int dev = current_device();
    std::lock_guard<std::mutex> lk(g_mu);
    release_all(g_cache[dev]);
}

size_t dev_free_memory() {
    const int dev = current_device();
    const auto now = std::chrono::steady_clock::now();
    {
        std::lock_guard<std::mutex> lk(g_mu);
        DeviceCache &c = g_cache[dev];
        if (c.free_mem && now - c.free_at < std::chrono::seconds(1)) return c.free_mem;
    }
    size_t f = 0, t = 0;
    MCE_CUDA(cudaMemGetInfo(&f, &t));
    std::lock_guard<std::mutex> lk(g_mu);
    DeviceCache &c = g_cache[dev];
    c.free_mem = f;
    c.free_at = now;
    return f;
}

void *host_pinned(size_t bytes, int slot) {
    const int dev = current_device();
    std::lock_guard<std::mutex> lk(g_mu);
    DeviceCache &c = g_cache[dev];
    if (c.pinned_bytes[slot] < bytes) {
        if (c.pinned[slot]) cudaFreeHost(c.pinned[slot]);
        c.pinned[slot] = nullptr;
        c.pinned_bytes[slot] = std::max<size_t>(bytes, 1 << 16);
        MCE_CUDA(cudaMallocHost(&c.pinned[slot], c.pinned_bytes[slot]));
    }
    return c.pinned[slot];
}

}  // namespace mce

extern "C" mce_status mce_empty_cache(int32_t device) {
    try {
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return MCE_ERR_INVALID;
        int prev = 0;
        cudaGetDevice(&prev);
        cudaSetDevice(device);
        mce::dev_empty_cache();
        cudaSetDevice(prev);
        return MCE_OK;
    } catch (...) {
        return MCE_ERR_CUDA;
    }
}
