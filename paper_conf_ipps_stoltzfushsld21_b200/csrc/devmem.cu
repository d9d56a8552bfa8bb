// devmem.cu -- the library's device-memory cache (a caching allocator over
// cudaMalloc, like torch's).  Rooms and plans allocate through dev_alloc; a
// freed block goes back to a per-device cache instead of cudaFree (which took
// 16 ms for the C4 hall's ~20 GB, and whose cost varied up to 0.6 s from run to
// run), and the next allocation of a similar size (best fit within 25 % + 1 MB)
// takes it back.  Callers free only blocks no pending work uses (setup and
// teardown paths synchronise first).  rafd_destroy trims the cache to half of
// the device's memory; an allocation that fails empties the cache and retries
// once; rafd_release_cached_memory() frees everything.  RAFD_POOL=0 disables
// caching (plain cudaMalloc / cudaFree).  A CUDA stream-ordered memory pool was
// measured first and not kept: its first-use allocations map memory eagerly
// (111 ms for K and two C4 fields against 1.2 ms with cudaMalloc).
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "internal.cuh"

namespace rafd {

namespace {
struct Block {
    void *p;
    size_t bytes;
};
struct Live {
    int dev;
    size_t bytes;
};
std::mutex mu;
std::vector<Block> cache[64];
size_t cached_bytes[64];
std::unordered_map<void *, Live> live;  // cached-capable allocations in use
}  // namespace

bool dev_cache_enabled()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("RAFD_POOL");
        v = !(e && strcmp(e, "0") == 0);
    }
    return v == 1;
}

void dev_cache_trim(int dev, size_t keep)
{
    if (dev < 0 || dev >= 64) return;
    std::lock_guard<std::mutex> lk(mu);
    auto &c = cache[dev];
    std::sort(c.begin(), c.end(), [](const Block &a, const Block &b) { return a.bytes < b.bytes; });
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != dev) cudaSetDevice(dev);
    while (!c.empty() && cached_bytes[dev] > keep) {
        cudaFree(c.back().p);
        cached_bytes[dev] -= c.back().bytes;
        c.pop_back();
    }
    if (cur != dev && cur >= 0) cudaSetDevice(cur);
}

cudaError_t dev_alloc(void **p, size_t bytes, bool cached)
{
    *p = nullptr;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    cached = cached && dev_cache_enabled() && dev < 64;
    if (cached) {
        std::lock_guard<std::mutex> lk(mu);
        auto &c = cache[dev];
        int best = -1;
        for (int i = 0; i < (int)c.size(); i++)
            if (c[i].bytes >= bytes && c[i].bytes <= bytes + bytes / 4 + (1u << 20) &&
                (best < 0 || c[i].bytes < c[best].bytes))
                best = i;
        if (best >= 0) {
            *p = c[best].p;
            live[*p] = {dev, c[best].bytes};
            cached_bytes[dev] -= c[best].bytes;
            c.erase(c.begin() + best);
            return cudaSuccess;
        }
    }
    e = cudaMalloc(p, bytes);
    if (e == cudaErrorMemoryAllocation && cached) {  // give the cache back and retry once
        cudaGetLastError();
        dev_cache_trim(dev, 0);
        e = cudaMalloc(p, bytes);
    }
    if (e != cudaSuccess) {
        *p = nullptr;
        return e;
    }
    if (cached) {
        std::lock_guard<std::mutex> lk(mu);
        live[*p] = {dev, bytes};
    }
    return cudaSuccess;
}

void dev_free(void *p)
{
    if (!p) return;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = live.find(p);
        if (it != live.end()) {
            cache[it->second.dev].push_back({p, it->second.bytes});
            cached_bytes[it->second.dev] += it->second.bytes;
            live.erase(it);
            return;
        }
    }
    cudaFree(p);
}

}  // namespace rafd
