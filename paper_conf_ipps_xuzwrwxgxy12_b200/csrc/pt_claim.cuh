// pt_claim.cuh -- work distribution shared by the persistent tracking kernels: CTA claims
// from the global work queue (one atomicAdd per claim) and 32-particle warp sub-chunks
// handed out through a shared-memory ticket word.  Replaces the paper's host-side
// segmentation and relaunch with on-device claims.
#pragma once
#include <cstdint>

#include "pt_internal.h"

namespace pt {

// CTA work distribution (REFILL kernel): s_work packs (CTA chunk index << 24 | tickets
// taken).  A warp takes ticket t: t < subs(chunk) -> sub-chunk t of the CTA chunk;
// t == subs -> this warp claims the next global chunk and publishes it; t > subs -> wait
// for the publication and retry.  Returns (seed index << 32 | first j) or kNoWork.
constexpr unsigned long long kNoWork = ~0ull;
constexpr unsigned long long kNoChunk = (1ull << 40) - 1;  // initial "empty" chunk id

// Number of 32-particle sub-chunks in claim unit `chunk`: either a slice of one seed
// (seeds_per_claim == 1), or seeds_per_claim whole consecutive seeds (in processing order)
// for the first group_chunks claims and one whole seed per claim after them (the tail:
// small last claims keep the CTAs' finishing times within about one seed of each other).
__device__ __forceinline__ uint32_t chunk_subs(unsigned long long chunk, const TrackArgs& a) {
    const uint32_t sps = (uint32_t)((a.P + kSub - 1) / kSub);  // sub-chunks per seed
    if (a.seeds_per_claim > 1) return chunk < a.group_chunks ? a.seeds_per_claim * sps : sps;
    const uint64_t k = chunk / a.chunks_per_seed;
    const uint64_t jbase = (chunk - k * a.chunks_per_seed) * (uint64_t)a.cta_chunk;
    const uint64_t cnt = a.P - jbase < a.cta_chunk ? a.P - jbase : a.cta_chunk;
    (void)sps;
    return (uint32_t)((cnt + kSub - 1) / kSub);
}

// (seed index << 32 | first j) of sub-chunk t of claim unit `chunk`
__device__ __forceinline__ unsigned long long chunk_sub(unsigned long long chunk, uint32_t t, const TrackArgs& a) {
    uint64_t k, j;
    if (a.seeds_per_claim > 1) {
        if (chunk < a.group_chunks) {
            const uint32_t sps = (uint32_t)((a.P + kSub - 1) / kSub);
            const uint32_t o = t / sps;
            k = chunk * a.seeds_per_claim + o;
            j = (uint64_t)(t - o * sps) * kSub;
        } else {  // tail: one seed per claim
            k = a.group_chunks * a.seeds_per_claim + (chunk - a.group_chunks);
            j = (uint64_t)t * kSub;
        }
    } else {
        k = chunk / a.chunks_per_seed;
        j = (chunk - k * a.chunks_per_seed) * (uint64_t)a.cta_chunk + (uint64_t)t * kSub;
    }
    PT_BOUND(a, k < a.nseeds);
    const uint32_t seed = a.order ? a.order[k] : (uint32_t)k;
    return ((unsigned long long)seed << 32) | j;
}

__device__ __forceinline__ unsigned long long cta_take(unsigned long long* s_work, const TrackArgs& a) {
    for (;;) {
        const unsigned long long old = atomicAdd(s_work, 1ull);
        const unsigned long long chunk = old >> 24;
        const uint32_t t = (uint32_t)(old & 0xFFFFFFull);
        uint32_t subs = 0;
        if (chunk != kNoChunk) {
            if (chunk >= a.total_chunks) return kNoWork;
            subs = chunk_subs(chunk, a);
        }
        if (t < subs) return chunk_sub(chunk, t, a);
        if (t == subs) {
            const unsigned long long c = atomicAdd(a.stats + kStatQueue, 1ull);
            atomicExch(s_work, (c << 24) | 1ull);
            if (c >= a.total_chunks) return kNoWork;
            return chunk_sub(c, 0u, a);
        }
        while ((*reinterpret_cast<volatile unsigned long long*>(s_work) >> 24) == chunk) __nanosleep(64);
    }
}

}  // namespace pt
