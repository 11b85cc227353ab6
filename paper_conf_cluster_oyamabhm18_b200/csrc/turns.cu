// turns.cu -- ordered split-K turn counters (deterministic BackwardFilter,
// dW = sum over samples, "only if each of the iterations is
// performed sequentially" does the micro-batched result keep its meaning).
//
// A BackwardFilter launch that splits the pixel reduction of one dw tile over
// several CTAs combines the partial tiles in split order: split s waits until
// the tile's counter holds tag(epoch, s - 1), adds its partial into dw (split
// 0 applies the user's beta) and publishes tag(epoch, s).  The counters are a
// static device pool (module memory, no cudaMalloc): each launch takes a fresh
// contiguous range of it and a process-unique epoch, so stale values from
// earlier launches never match and no reset pass is needed.
#include <cuda_runtime.h>

#include <atomic>
#include <mutex>

#include "mucudnn_internal.h"

namespace mucu {

constexpr int64_t kTurnPool = 1 << 18;  // counters (8 B each) per device
__device__ unsigned long long g_turn_pool[kTurnPool];

namespace {
std::atomic<unsigned long long> g_epoch{0};
std::mutex g_turn_mu;
int64_t g_turn_next[64] = {0};
unsigned long long* g_turn_base[64] = {nullptr};
}  // namespace

int alloc_turns(int64_t count, TurnRange* out) {
    out->ctr = nullptr;
    out->epoch = 0;
    if (count <= 0) return 0;
    if (count > kTurnPool) return (int)cudaErrorInvalidValue;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e) return (int)e;
    if (dev < 0 || dev >= 64) return (int)cudaErrorInvalidDevice;
    std::lock_guard<std::mutex> lk(g_turn_mu);
    if (!g_turn_base[dev]) {
        void* p = nullptr;
        e = cudaGetSymbolAddress(&p, g_turn_pool);
        if (e) return (int)e;
        g_turn_base[dev] = (unsigned long long*)p;
    }
    if (g_turn_next[dev] + count > kTurnPool) g_turn_next[dev] = 0;  // ring: ranges stay contiguous
    out->ctr = g_turn_base[dev] + g_turn_next[dev];
    g_turn_next[dev] += count;
    out->epoch = g_epoch.fetch_add(1, std::memory_order_relaxed) + 1;
    return 0;
}

}  // namespace mucu
