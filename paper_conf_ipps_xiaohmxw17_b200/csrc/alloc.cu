// Caching device allocator for the library's own arrays (matrix, preconditioner, PCG workspace,
// assembly temporaries).
//
// The open-close loop of DDA rebuilds K from the current contacts in every loop,
// so dda_build_matrix / dda_matrix_free run once per solve.  Measured on B200 with the stream-ordered
// pool (cudaMallocAsync, release threshold = max): the 13 allocations of one 1M-block build took
// 1.7 to 71 ms of host time, with the GPU idle.  This allocator keeps freed blocks in per-device
// size-ordered free lists and hands them back without any CUDA call, so a rebuild of a same-sized
// system allocates nothing.
//
//  * Sizes are rounded up to 512 B below 1 MiB and to 2 MiB above; a cached block is reused for a
//    request of at most its size and at least 3/4 of it (plus one 2 MiB granule).
//  * Stream order: dev_free_on(p, s) records an event on s; a later dev_alloc on stream t that
//    reuses the block makes t wait for that event (the semantics of cudaFreeAsync/cudaMallocAsync).
//    dev_free(p) frees on the legacy default stream.
//  * Out of memory: the cached blocks of the device are released (after a device synchronise)
//    and the cudaMalloc is retried once.
//  * dda_memory_release() returns every cached block to the driver.
#include <cstdint>
#include <map>
#include <mutex>
#include <unordered_map>

#include "dda_internal.cuh"

namespace dda {
namespace {

struct Blk {
    void* p = nullptr;
    size_t size = 0;
    int dev = 0;
    cudaEvent_t ev = nullptr;   // recorded at the last free
};

struct Cache {
    std::mutex mu;
    std::unordered_map<void*, Blk> live;
    std::map<int, std::multimap<size_t, Blk>> free_by_dev;
    int64_t cached_bytes = 0;
};

Cache& cache() {
    static Cache* c = new Cache();   // never destroyed: frees may run during static destruction
    return *c;
}

size_t round_size(size_t bytes) {
    if (bytes == 0) bytes = 1;
    const size_t small = size_t(1) << 20, gran = size_t(2) << 20;
    if (bytes < small) return (bytes + 511) & ~size_t(511);
    return (bytes + gran - 1) & ~(gran - 1);
}

// releases the device's cached blocks (caller holds the lock)
void release_locked(Cache& c, int dev) {
    auto it = c.free_by_dev.find(dev);
    if (it == c.free_by_dev.end() || it->second.empty()) return;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(dev);
    cudaDeviceSynchronize();
    for (auto& kv : it->second) {
        if (kv.second.ev) cudaEventDestroy(kv.second.ev);
        cudaFree(kv.second.p);
        c.cached_bytes -= (int64_t)kv.second.size;
    }
    it->second.clear();
    cudaSetDevice(prev);
}

}  // namespace

cudaError_t dev_alloc(void** p, size_t bytes, cudaStream_t st) {
    *p = nullptr;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const size_t want = round_size(bytes);
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    auto& fl = c.free_by_dev[dev];
    auto it = fl.lower_bound(want);
    if (it != fl.end() && it->first <= want + want / 3 + (size_t(2) << 20)) {
        Blk b = it->second;
        fl.erase(it);
        c.cached_bytes -= (int64_t)b.size;
        if (b.ev) cudaStreamWaitEvent(st, b.ev, 0);
        c.live[b.p] = b;
        *p = b.p;
        return cudaSuccess;
    }
    void* q = nullptr;
    e = cudaMalloc(&q, want);
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();          // reset the last-error state of the failed call
        release_locked(c, dev);
        e = cudaMalloc(&q, want);
    }
    if (e != cudaSuccess) return e;
    Blk b;
    b.p = q;
    b.size = want;
    b.dev = dev;
    c.live[q] = b;
    *p = q;
    return cudaSuccess;
}

void dev_free_on(void* p, cudaStream_t st) {
    if (!p) return;
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    auto it = c.live.find(p);
    if (it == c.live.end()) return;   // not ours (never happens for library arrays)
    Blk b = it->second;
    c.live.erase(it);
    int prev = 0;
    cudaGetDevice(&prev);
    if (prev != b.dev) cudaSetDevice(b.dev);
    if (!b.ev) cudaEventCreateWithFlags(&b.ev, cudaEventDisableTiming);
    if (b.ev) cudaEventRecord(b.ev, st);
    if (prev != b.dev) cudaSetDevice(prev);
    c.free_by_dev[b.dev].emplace(b.size, b);
    c.cached_bytes += (int64_t)b.size;
}

void dev_free(void* p) { dev_free_on(p, 0); }

}  // namespace dda

// Returns every cached (freed) device block of every device to the driver.
extern "C" void dda_memory_release(void) {
    using namespace dda;
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    for (auto& kv : c.free_by_dev) release_locked(c, kv.first);
}

// Bytes held in the free lists (cached, not in use) across devices.
extern "C" int64_t dda_memory_cached(void) {
    using namespace dda;
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    return c.cached_bytes;
}
