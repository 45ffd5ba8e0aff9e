// alloc.cu -- device block cache for allocations that outlive one API call
// (the index arrays, the hash table, device-resident results).
//
// Those blocks are freed by a later call, possibly from another thread or on
// another stream than the one they were allocated on; stream-ordered pool
// memory freed that way is not reused by the next stream-ordered allocation
// and the pool maps fresh pages every time (measured: +20 ms per index
// build at 1.4 GB).  Freed blocks are therefore kept here and handed out
// again by size (best fit within 2x).  Callers free only after the device has
// finished using the block (dts_free_* synchronise first).
#include <map>
#include <mutex>
#include <unordered_map>

#include "internal.cuh"

namespace dts {
namespace {

constexpr size_t GRAIN = size_t(2) << 20;    // 2 MiB granules

struct Cache {
    std::mutex mu;
    std::multimap<size_t, void*> free_blocks[64];          // per device: size -> ptr
    std::unordered_map<void*, std::pair<int, size_t>> live;  // ptr -> (device, size)
    size_t cached[64] = {0};
};

Cache& cache() {
    static Cache* c = new Cache();   // never destroyed: frees may run at exit
    return *c;
}

void release_free_blocks(Cache& c, int dev) {
    for (auto& kv : c.free_blocks[dev]) cudaFree(kv.second);
    c.free_blocks[dev].clear();
    c.cached[dev] = 0;
}

}  // namespace

void* cache_alloc(size_t bytes) {
    int dev = 0;
    DTS_CUDA(cudaGetDevice(&dev));
    if (dev < 0 || dev >= 64) throw Error(DTS_ENOTSUP, "device ordinal >= 64");
    const size_t sz = ((bytes + GRAIN - 1) / GRAIN) * GRAIN;
    Cache& c = cache();
    {
        std::lock_guard<std::mutex> lk(c.mu);
        auto it = c.free_blocks[dev].lower_bound(sz);
        if (it != c.free_blocks[dev].end() && it->first <= 2 * sz) {
            void* p = it->second;
            const size_t have = it->first;
            c.free_blocks[dev].erase(it);
            c.cached[dev] -= have;
            c.live[p] = {dev, have};
            return p;
        }
    }
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, sz);
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        std::lock_guard<std::mutex> lk(c.mu);
        DTS_CUDA(cudaDeviceSynchronize());
        release_free_blocks(c, dev);
        e = cudaMalloc(&p, sz);
    }
    if (e != cudaSuccess) {
        cudaGetLastError();
        throw Error(e == cudaErrorMemoryAllocation ? DTS_ENOMEM : DTS_ECUDA,
                    std::string("cudaMalloc: ") + cudaGetErrorString(e));
    }
    std::lock_guard<std::mutex> lk(c.mu);
    c.live[p] = {dev, sz};
    return p;
}

void cache_free(void* p) {
    if (!p) return;
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    auto it = c.live.find(p);
    if (it == c.live.end()) return;            // not ours
    const int dev = it->second.first;
    const size_t sz = it->second.second;
    c.live.erase(it);
    c.free_blocks[dev].emplace(sz, p);
    c.cached[dev] += sz;
}

int cache_device(void* p) {
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    auto it = c.live.find(p);
    return it == c.live.end() ? -1 : it->second.first;
}

bool cache_owns(void* p) {
    Cache& c = cache();
    std::lock_guard<std::mutex> lk(c.mu);
    return c.live.count(p) != 0;
}

}  // namespace dts
