// pt_kernels.cu -- sm_100a kernels of the probabilistic-streamlining hot path.
//
//   track_kernel   : particle stepping (Algorithm 1's inner loop, with the
//                    semantics of P:L98-121), persistent warps + lane refill (REFILL) or
//                    one particle per lane without refill (the paper's "Extreme case 1",
//                    P:L199-201; ablation)
//   repack_kernel  : canonical sample volumes -> one record per (voxel, sample)
//   map_sum_kernel : sum of the uint32 map (overflow detection, R17)
//   gather_bench   : random-record gather micro-benchmark (roofline denominator)
//
// Design notes: one lane owns one particle at a time; particles are
// claimed in chunks of kChunk from a global atomic work queue and dead lanes are refilled
// with a ballot/popc prefix at the start of every round, so the warp stays converged while
// path lengths are exponentially distributed.  A round is 3 steps: one
// Philox block per round supplies the three sample indices (R16).  The gather of the next
// step's record doubles as the mask test of the candidate voxel (sentinel records, R11);
// the third step's gather is deferred to the next round's start, where it is issued by
// the same instruction as the first gather of freshly refilled lanes.
#include <cuda_runtime.h>
#include <cub/device/device_radix_sort.cuh>

#include <cstdint>

#include "pt_device.cuh"
#include "pt_internal.h"

#ifndef PT_MIN_BLOCKS
#define PT_MIN_BLOCKS 1
#endif
#ifndef PT_MAP_HINT
#define PT_MAP_HINT 0  // 1: REDs carry an L2 evict_last policy (measured: no effect)
#endif
#ifndef PT_MAP_PERSIST
#define PT_MAP_PERSIST 0  // 1: persisting L2 access-policy window over the map (measured: no effect)
#endif
#ifndef PT_MAP_CACHE
#define PT_MAP_CACHE 0      // entries of the per-CTA shared-memory count cache (power of 2; 0 = off)
#endif

namespace pt {

enum { kEndMask = 0, kEndCurv = 1, kEndMaxlen = 2 };

// Per-CTA shared-memory cache of visitation counts (REFILL kernel).  Entry = (voxel+1) << 32
// | count; direct-mapped by a multiplicative hash.  A flush adds to the entry of its voxel
// or replaces a different voxel's entry, whose count then goes to the global map with one
// RED; the CTA drains the table at exit.  Integer sums commute, so the map is unchanged.
constexpr uint32_t kMapCache = PT_MAP_CACHE;

__device__ __forceinline__ void cache_add(unsigned long long* tab, uint32_t* map, uint32_t v, uint32_t c) {
    constexpr uint32_t kBits = kMapCache > 1 ? 31 - __builtin_clz(kMapCache) : 0;
    const uint32_t h = kBits ? (v * 0x9E3779B1u) >> (32 - kBits) : 0u;
    unsigned long long* e = tab + h;
    const uint32_t key = v + 1u;
    unsigned long long old = *reinterpret_cast<volatile unsigned long long*>(e);
    for (;;) {
        const uint32_t ok = (uint32_t)(old >> 32), oc = (uint32_t)old;
        const bool same = ok == key && oc < 0x80000000u;
        const unsigned long long want = same ? old + c : (((unsigned long long)key << 32) | c);
        const unsigned long long prev = atomicCAS(e, old, want);
        if (prev == old) {
            if (!same && ok != 0u) atomicAdd(map + (ok - 1u), oc);
            return;
        }
        old = prev;
    }
}

// CTA work distribution (REFILL kernel): s_work packs (CTA chunk index << 24 | tickets
// taken).  A warp takes ticket t: t < subs(chunk) -> sub-chunk t of the CTA chunk;
// t == subs -> this warp claims the next global chunk and publishes it; t > subs -> wait
// for the publication and retry.  Returns (seed index << 32 | first j) or kNoWork.
constexpr unsigned long long kNoWork = ~0ull;
constexpr unsigned long long kNoChunk = (1ull << 40) - 1;  // initial "empty" chunk id

// Number of 32-particle sub-chunks in claim unit `chunk`: either a slice of one seed
// (seeds_per_claim == 1) or seeds_per_claim whole consecutive seeds (in processing order).
__device__ __forceinline__ uint32_t chunk_subs(unsigned long long chunk, const TrackArgs& a) {
    const uint32_t sps = (uint32_t)((a.P + kSub - 1) / kSub);  // sub-chunks per seed
    if (a.seeds_per_claim > 1) {
        const uint64_t kb = chunk * a.seeds_per_claim;
        const uint64_t nk = a.nseeds - kb < a.seeds_per_claim ? a.nseeds - kb : a.seeds_per_claim;
        return (uint32_t)nk * sps;
    }
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
        const uint32_t sps = (uint32_t)((a.P + kSub - 1) / kSub);
        const uint32_t o = t / sps;
        k = chunk * a.seeds_per_claim + o;
        j = (uint64_t)(t - o * sps) * kSub;
    } else {
        k = chunk / a.chunks_per_seed;
        j = (chunk - k * a.chunks_per_seed) * (uint64_t)a.cta_chunk + (uint64_t)t * kSub;
    }
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

// OUT: per-particle outputs or polylines are recorded (compiled out of the bench path).
template <int F, bool HALF, bool REFILL, bool OUT>
__global__ void __launch_bounds__(REFILL ? kThreads : kSimpleThreads, PT_MIN_BLOCKS)
track_kernel(const __grid_constant__ TrackArgs a) {
    using R = Rec<F, HALF>;
    constexpr int RB = R::kBytes;
    constexpr int TPB = REFILL ? kThreads : kSimpleThreads;
    // rarely used state lives in shared memory to keep the hot loop's register count low
    __shared__ unsigned long long s_li[TPB];     // particle index of this call (outputs)
    __shared__ uint32_t s_q[TPB / 32][3];        // per-warp sub-chunk: seed, next j, end j
    __shared__ unsigned long long s_work;        // CTA chunk + tickets (see cta_take)
#if defined(PT_DIAG_RED) && PT_DIAG_RED == 1
    __shared__ uint32_t s_diag[1024];
#endif
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t wib = threadIdx.x >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    extern __shared__ unsigned long long s_cache[];  // kMapCache entries when REFILL && map
    constexpr bool kCache = REFILL && kMapCache > 0;
    const bool use_cache = kCache && a.map != nullptr;
    const bool has_map = a.map != nullptr;
    // privatised map: CTA b adds into copy b % map_copies (no cross-SM contention on the
    // hot lines near the seeds; the copies are summed by map_combine_kernel)
    uint32_t* const map = has_map ? a.map + (size_t)(blockIdx.x % a.map_copies) *
                                                  ((size_t)a.nx * a.ny * a.nz)
                                  : nullptr;
    const uint64_t map_pol = PT_MAP_HINT ? l2_evict_last_policy() : 0ull;
    if (threadIdx.x == 0) s_work = kNoChunk << 24;
    if constexpr (kCache) {
        if (use_cache)
            for (uint32_t i = threadIdx.x; i < kMapCache; i += TPB) s_cache[i] = 0ull;
    }
    __syncthreads();

    // ---- per-lane particle state
    bool alive = false;   // lane holds a particle in flight
    bool pend = false;    // the round's 3rd candidate step waits for the next round's gather
    float qx = 0.f, qy = 0.f, qz = 0.f;   // committed position, centred coordinates (R10)
    float px = 0.f, py = 0.f, pz = 0.f;   // direction of the last (candidate) step
    uint32_t gvox = 0;    // voxel read by the round-start gather (seed or pending candidate)
    int n = 0;            // committed steps
    uint64_t pid = 0;     // global particle id = seed_id * P + j (RNG key, R16)
    uint32_t run_vox = 0, run_cnt = 0;  // run-length merge of consecutive visits
    uint32_t sfix = 0;    // paper mode (NEXT-1): the particle's sample volume, j mod S
    R rv;                 // record of the current step
    uint4 W = make_uint4(0u, 0u, 0u, 0u);

    // ---- per-lane counters (a lane never sees 2^32 steps in one launch)
    uint32_t my_steps = 0, my_particles = 0, my_active = 0, rounds = 0;
    bool exhausted = false;  // warp-uniform
    if (lane == 0) {
        s_q[wib][0] = 0u;
        s_q[wib][1] = 0u;
        s_q[wib][2] = 0u;
    }
    __syncwarp();

    int why = -1;  // >= 0: the particle ended with this reason; outputs pending (finish())

    auto red = [&](uint32_t v, uint32_t c) {
        if (kCache && use_cache) cache_add(s_cache, map, v, c);
        else atomicAdd(map + v, c);  // no return value used -> RED
    };
    // a termination only records the reason; the outputs are written once per round for
    // all ended lanes at the top of the loop (one divergent block instead of one per site)
    auto end = [&](int w) {
        why = w;
        alive = false;
        pend = false;
    };
    // SetEndPoint()
    auto finish = [&]() {
        if (OUT && (a.o_nsteps || a.o_reason || a.o_end)) {
            const uint64_t li = s_li[threadIdx.x];
            if (a.o_nsteps) a.o_nsteps[li] = (uint16_t)n;
            if (a.o_reason) a.o_reason[li] = (uint8_t)why;
            if (a.o_end) {
                float* e = a.o_end + 3 * li;
                e[0] = __fadd_rn(qx, a.fcx);
                e[1] = __fadd_rn(qy, a.fcy);
                e[2] = __fadd_rn(qz, a.fcz);
            }
        }
        if (has_map && run_cnt) red(run_vox, run_cnt);
        run_cnt = 0;
        my_steps += (uint32_t)n;
        my_particles += 1u;
        why = -1;
    };
    // commit a step (lanes with c): new position, one visit of the new voxel (R13);
    // consecutive visits of the same voxel are merged (run length) and flushed with a
    // predicated RED when the voxel changes.  Straight-line, no branch.
    auto commit_if = [&](bool c, float x, float y, float z, uint32_t v) {
        qx = c ? x : qx;
        qy = c ? y : qy;
        qz = c ? z : qz;
        n += c ? 1 : 0;
        if (has_map) {
            const bool change = v != run_vox;
            if (kCache && use_cache) {
                if (c && change && run_cnt != 0u) red(run_vox, run_cnt);
            } else {
#if defined(PT_DIAG_RED) && PT_DIAG_RED == 1  // diagnostic builds only (wrong maps)
                if (c && change && run_cnt != 0u) atomicAdd(&s_diag[run_vox & 1023u], run_cnt);
#elif defined(PT_DIAG_RED) && PT_DIAG_RED == 2
                red_add_if(c && change && run_cnt != 0u, a.map + ((run_vox & 4095u) + blockIdx.x * 4096u), run_cnt);
#else
                if (PT_MAP_HINT) red_add_if_hint(c && change && run_cnt != 0u, map + run_vox, run_cnt, map_pol);
                else red_add_if(c && change && run_cnt != 0u, map + run_vox, run_cnt);
#endif
            }
            run_cnt = c ? (change ? 1u : run_cnt + 1u) : run_cnt;
            run_vox = c ? v : run_vox;
        }
        if (OUT && a.o_paths && c && n < a.path_stride) {
            float* pp = a.o_paths + (s_li[threadIdx.x] * (uint64_t)a.path_stride + (uint64_t)n) * 3u;
            pp[0] = __fadd_rn(qx, a.fcx);
            pp[1] = __fadd_rn(qy, a.fcy);
            pp[2] = __fadd_rn(qz, a.fcz);
        }
    };
    // GetStartPoint(): centred seed position, seed voxel (R10, R12)
    auto start = [&](uint64_t si, uint64_t j) {
        const uint64_t li = si * a.P + j;
        if (OUT) s_li[threadIdx.x] = li;
        const uint64_t sid = a.seed_ids ? a.seed_ids[si] : si;
        pid = sid * a.P + j;
        sfix = (uint32_t)(j % a.S);
        qx = __fsub_rn(a.seeds[3 * si + 0], a.fcx);
        qy = __fsub_rn(a.seeds[3 * si + 1], a.fcy);
        qz = __fsub_rn(a.seeds[3 * si + 2], a.fcz);
        n = 0;
        pend = false;
        run_cnt = 0;
        alive = true;
        if (OUT && a.o_paths) {
            float* pp = a.o_paths + li * (uint64_t)a.path_stride * 3u;
            pp[0] = __fadd_rn(qx, a.fcx);
            pp[1] = __fadd_rn(qy, a.fcy);
            pp[2] = __fadd_rn(qz, a.fcz);
        }
        const int ix = axis_index(qx, a.cx), iy = axis_index(qy, a.cy), iz = axis_index(qz, a.cz);
        if ((unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny &&
            (unsigned)iz < (unsigned)a.nz) {
            gvox = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
        } else {
            end(kEndMask);  // seed outside the volume (R12): finished right away, so the
            finish();       // refill loop may hand this lane another particle
        }
    };

    if (!REFILL) {
        const uint64_t g = (uint64_t)blockIdx.x * TPB + threadIdx.x;
        if (g < a.nparticles) {
            const uint64_t si = g / a.P;
            start(si, g - si * a.P);
        }
    }

    for (;;) {
        if (why >= 0) finish();  // particles that ended during the previous round

        // ------------------------------------------------ lane refill (replaces the
        // paper's CPU Reduction()/segment relaunch)
        if (REFILL) {
            uint32_t need = __ballot_sync(kFull, !alive);
            if (need != 0u && !exhausted) {
                uint32_t cseed = s_q[wib][0], cnext = s_q[wib][1], cend = s_q[wib][2];
                while (need != 0u) {
                    if (cnext == cend) {
                        unsigned long long r = 0;
                        if (lane == 0) r = cta_take(&s_work, a);
                        r = __shfl_sync(kFull, r, 0);
                        if (r == kNoWork) {
                            exhausted = true;
                            break;
                        }
                        cseed = (uint32_t)(r >> 32);
                        cnext = (uint32_t)r;
                        const uint64_t e = (uint64_t)cnext + kSub;
                        cend = (uint32_t)(e < a.P ? e : a.P);
                    }
                    const uint32_t avail = cend - cnext;
                    const uint32_t rank = __popc(need & lt_mask);
                    if (!alive && rank < avail) start(cseed, (uint64_t)(cnext + rank));
                    const uint32_t cnt = (uint32_t)__popc(need);
                    cnext += cnt < avail ? cnt : avail;
                    need = __ballot_sync(kFull, !alive);
                }
                __syncwarp();
                if (lane == 0) {
                    s_q[wib][0] = cseed;
                    s_q[wib][1] = cnext;
                    s_q[wib][2] = cend;
                }
                __syncwarp();
            }
        }
        if (!__any_sync(kFull, alive)) break;
        rounds += 1u;

        // ------------------------------------------------ round start: one Philox block,
        // gather of (pending candidate | seed) voxel = mask test + first step's record.
        // Straight-line code: every lane computes, only live lanes load / commit.
        {
            const uint32_t t0 = (uint32_t)n + (pend ? 1u : 0u);  // a multiple of 3
            W = philox4x32_10(make_uint4(t0 / 3u, (uint32_t)pid, (uint32_t)(pid >> 32), 0u),
                              a.key0, a.key1);
            const uint32_t s0 = a.sample_mode ? sfix : sample_of(W.x, a.S);
            ldg_record_if<RB>(alive, a.rec + ((uint64_t)gvox * a.S + s0) * RB, rv.w);
            // seed outside the mask (R12) or pending candidate rejected (R11)
            const bool outside = alive && rv.outside();
            why = outside ? kEndMask : why;
            alive = alive && !outside;
            // accepted candidate: recomputed bit-identically from (q, d) instead of kept
            commit_if(pend && !outside, __fadd_rn(qx, __fmul_rn(a.step, px)),
                      __fadd_rn(qy, __fmul_rn(a.step, py)), __fadd_rn(qz, __fmul_rn(a.step, pz)), gvox);
            pend = false;
        }

        // ------------------------------------------------ three steps
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            my_active += alive ? 1u : 0u;
            const bool first = n == 0;
            // choose the fibre closest to the previous direction: eligible iff
            // f_j > fib_thr (R7), strict >, lowest j wins (R8); the first step takes fibre 0
            // (R5).  "Interpolation()" of Alg. 1 = this sample's record at the voxel (R2).
            float vx, vy, vz, f0;
            rv.fibre(0, vx, vy, vz, f0);
            float bc = __fadd_rn(__fadd_rn(__fmul_rn(vx, px), __fmul_rn(vy, py)), __fmul_rn(vz, pz));
            float best = f0 > a.fib_thr ? fabsf(bc) : -1.f;
#pragma unroll
            for (int j = 1; j < F; ++j) {
                float ux, uy, uz, fu;
                rv.fibre(j, ux, uy, uz, fu);
                const float cj = __fadd_rn(__fadd_rn(__fmul_rn(ux, px), __fmul_rn(uy, py)), __fmul_rn(uz, pz));
                const bool pick = !first && fu > a.fib_thr && fabsf(cj) > best;
                best = pick ? fabsf(cj) : best;
                bc = pick ? cj : bc;
                vx = pick ? ux : vx;
                vy = pick ? uy : vy;
                vz = pick ? uz : vz;
            }
            // maximum angle, measured by the dot product (R4); orientation
            // kept (R9); first step: sign = top bit of word 3 of block 0 (R6, R16)
            const bool curv_ok = first || fabsf(bc) > a.curv_thr;
            const bool neg = first ? (W.w >> 31) != 0u : !(bc > 0.f);
            // StepToNextPoint(): q' = q + h * (sign * v), no FMA
            const float dx = neg ? -vx : vx, dy = neg ? -vy : vy, dz = neg ? -vz : vz;
            const float nqx = __fadd_rn(qx, __fmul_rn(a.step, dx));
            const float nqy = __fadd_rn(qy, __fmul_rn(a.step, dy));
            const float nqz = __fadd_rn(qz, __fmul_rn(a.step, dz));
            const int ix = axis_index(nqx, a.cx), iy = axis_index(nqy, a.cy), iz = axis_index(nqz, a.cz);
            const bool inb = (unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny &&
                             (unsigned)iz < (unsigned)a.nz;
            const uint32_t v = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
            // stop criteria in order: maximum steps (R14), angle, volume (R11)
            const bool maxed = n == a.max_steps;
            const bool go = alive && !maxed && curv_ok && inb;
            why = (alive && !go) ? (maxed ? kEndMaxlen : (!curv_ok ? kEndCurv : kEndMask)) : why;
            alive = go;
            px = go ? dx : px;
            py = go ? dy : py;
            pz = go ? dz : pz;
            if (k < 2) {
                const uint32_t w = (k == 0) ? W.y : W.z;
                const uint32_t sk = a.sample_mode ? sfix : sample_of(w, a.S);
                ldg_record_if<RB>(go, a.rec + ((uint64_t)v * a.S + sk) * RB, rv.w);
                const bool outside = go && rv.outside();  // candidate outside the mask (R11)
                why = outside ? kEndMask : why;
                alive = go && !outside;
                commit_if(alive, nqx, nqy, nqz, v);
            } else {
                pend = go;  // next round's start gathers and tests it
                gvox = go ? v : gvox;
            }
        }
    }

    // ---- drain the count cache
    if constexpr (kCache) {
        if (use_cache) {
            __syncthreads();
            for (uint32_t i = threadIdx.x; i < kMapCache; i += TPB) {
                const unsigned long long e = s_cache[i];
                if (e >> 32) atomicAdd(map + ((uint32_t)(e >> 32) - 1u), (uint32_t)e);
            }
        }
    }

    // ---- counters: one atomic per warp
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        my_steps += __shfl_xor_sync(kFull, my_steps, o);
        my_particles += __shfl_xor_sync(kFull, my_particles, o);
        my_active += __shfl_xor_sync(kFull, my_active, o);
    }
    if (lane == 0) {
        atomicAdd(a.stats + kStatSteps, (unsigned long long)my_steps);
        atomicAdd(a.stats + kStatParticles, (unsigned long long)my_particles);
        atomicAdd(a.stats + kStatLaneActive, (unsigned long long)my_active);
        atomicAdd(a.stats + kStatLaneSlots, (unsigned long long)rounds * 3ull * 32ull);
    }
}

// ------------------------------------------------------------------------- repack
// Canonical [F][S][Z][Y][X](x3) sample volumes -> rec[vox][s] (one thread per record,
// s fastest so the record stores are coalesced).  Voxels outside the mask get the
// sentinel f0 = all-ones; non-finite values inside the mask are counted in *bad.
template <bool HALF>
__global__ void repack_kernel(const void* __restrict__ dyads, const void* __restrict__ fr,
                              const uint8_t* __restrict__ mask, uint8_t* __restrict__ rec,
                              int64_t V, int S, int F, int RB, unsigned long long* bad) {
    const int64_t total = V * (int64_t)S;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t vox = i / S;
        const int s = (int)(i - vox * S);
        uint32_t w[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) w[k] = 0u;
        const bool inside = mask[vox] != 0;
        bool ok = true;
        for (int j = 0; j < F; ++j) {
            const int64_t e = ((int64_t)j * S + s) * V + vox;
            if (HALF) {
                const uint16_t* d = static_cast<const uint16_t*>(dyads);
                const uint16_t* f = static_cast<const uint16_t*>(fr);
                const uint16_t x = d[3 * e], y = d[3 * e + 1], z = d[3 * e + 2], ff = f[e];
                ok = ok && ((x & 0x7C00u) != 0x7C00u) && ((y & 0x7C00u) != 0x7C00u) &&
                     ((z & 0x7C00u) != 0x7C00u) && ((ff & 0x7C00u) != 0x7C00u);
                w[2 * j] = (uint32_t)x | ((uint32_t)y << 16);
                w[2 * j + 1] = (uint32_t)z | ((uint32_t)ff << 16);
            } else {
                const float* d = static_cast<const float*>(dyads);
                const float* f = static_cast<const float*>(fr);
                const float x = d[3 * e], y = d[3 * e + 1], z = d[3 * e + 2], ff = f[e];
                ok = ok && isfinite(x) && isfinite(y) && isfinite(z) && isfinite(ff);
                w[4 * j] = __float_as_uint(x);
                w[4 * j + 1] = __float_as_uint(y);
                w[4 * j + 2] = __float_as_uint(z);
                w[4 * j + 3] = __float_as_uint(ff);
            }
        }
        if (!inside) {
            if (HALF) w[1] |= 0xFFFF0000u;
            else w[3] = 0xFFFFFFFFu;
        } else if (!ok) {
            atomicAdd(bad, 1ull);
        }
        uint8_t* out = rec + i * RB;
        if (RB == 8) {
            *reinterpret_cast<uint2*>(out) = make_uint2(w[0], w[1]);
        } else {
            for (int k = 0; k < RB / 16; ++k)
                reinterpret_cast<uint4*>(out)[k] = make_uint4(w[4 * k], w[4 * k + 1], w[4 * k + 2], w[4 * k + 3]);
        }
    }
}

// ------------------------------------------------------------------------- seed order
// Morton key of the seed's voxel (10 bits per axis; coordinates clamped to [0, 1023]),
// with the input index in the low 32 bits so the sort is a total order.
__device__ __forceinline__ uint64_t spread3(uint32_t v) {
    uint64_t x = v & 0x3FFu;
    x = (x | (x << 16)) & 0x030000FFull;
    x = (x | (x << 8)) & 0x0300F00Full;
    x = (x | (x << 4)) & 0x030C30C3ull;
    x = (x | (x << 2)) & 0x09249249ull;
    return x;
}

__global__ void seed_keys_kernel(const float* __restrict__ seeds, uint64_t n, uint32_t* keys,
                                 uint32_t* idx) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t c[3];
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            const float x = seeds[3 * i + a];
            c[a] = x <= 0.f ? 0u : (x >= 1023.f ? 1023u : (uint32_t)x);
        }
        keys[i] = (uint32_t)(spread3(c[0]) | (spread3(c[1]) << 1) | (spread3(c[2]) << 2));
        idx[i] = (uint32_t)i;
    }
}

size_t seed_order_temp_bytes(uint64_t nseeds) {
    size_t bytes = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, bytes, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                    (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)nseeds, 0, 30);
    return bytes;
}

cudaError_t launch_seed_order(const float* seeds, uint64_t nseeds, uint32_t* keys, uint32_t* keys_out,
                              uint32_t* idx, uint32_t* perm, void* temp, size_t temp_bytes, cudaStream_t st) {
    if (nseeds == 0) return cudaSuccess;
    uint64_t blocks = (nseeds + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    seed_keys_kernel<<<(unsigned)blocks, 256, 0, st>>>(seeds, nseeds, keys, idx);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    // stable radix sort on the 30-bit Morton code: ties keep the input order
    return cub::DeviceRadixSort::SortPairs(temp, temp_bytes, keys, keys_out, idx, perm, (int)nseeds, 0, 30, st);
}

// ------------------------------------------------------------------------- map combine
__global__ void map_combine_kernel(const uint32_t* __restrict__ copies, uint32_t ncopies, int64_t V,
                                   uint32_t* __restrict__ out, bool accumulate) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t s = accumulate ? out[i] : 0u;
        for (uint32_t c = 0; c < ncopies; ++c) s += __ldg(copies + (int64_t)c * V + i);
        out[i] = s;
    }
}

cudaError_t launch_map_combine(const uint32_t* copies, uint32_t ncopies, int64_t V, uint32_t* out,
                               bool accumulate, cudaStream_t st) {
    int64_t blocks = (V + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (blocks < 1) blocks = 1;
    map_combine_kernel<<<(unsigned)blocks, 256, 0, st>>>(copies, ncopies, V, out, accumulate);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------- map sum
__global__ void map_sum_kernel(const uint32_t* __restrict__ map, int64_t V, unsigned long long* out) {
    unsigned long long s = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += (int64_t)gridDim.x * blockDim.x)
        s += map[i];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

// ------------------------------------------------------------------------- gather bench
// Uniformly random record-aligned reads, 8 independent loads in flight per thread.
template <int RB>
__global__ void __launch_bounds__(256) gather_bench_kernel(const uint8_t* __restrict__ buf, uint64_t nrec,
                                                           uint32_t iters, uint32_t seed, uint32_t* sink) {
    uint32_t x = (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u ^ seed;
    uint32_t acc = 0;
    for (uint32_t it = 0; it < iters; it += 8) {
        uint32_t w[8][RB / 4 > 16 ? 16 : RB / 4];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            x ^= x << 13;
            x ^= x >> 17;
            x ^= x << 5;
            const uint64_t r = ((uint64_t)x * nrec) >> 32;
            ldg_record<RB>(buf + r * RB, w[u]);
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) acc ^= w[u][0] ^ w[u][RB / 4 - 1];
    }
    if (acc == 0x9E3779B9u) sink[0] = acc;
}

// ------------------------------------------------------------------------- launchers
template <int F, bool HALF, bool REFILL, bool OUT>
static cudaError_t launch_t(const TrackArgs& a, int num_sms, cudaStream_t st) {
    auto k = track_kernel<F, HALF, REFILL, OUT>;
    constexpr int TPB = REFILL ? kThreads : kSimpleThreads;
    if (a.nparticles == 0) return cudaSuccess;
    const size_t dyn = (REFILL && kMapCache > 0 && a.map) ? kMapCache * sizeof(unsigned long long) : 0;
    unsigned grid;
    if (REFILL) {
        int per_sm = 0;
        cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)(kMapCache * sizeof(unsigned long long)));
        if (e == cudaSuccess)  // prefer L1 over shared memory: records are gathered through L1
            e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, kMapCache ? -1 : 0);
        if (e != cudaSuccess) return e;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, TPB, dyn);
        if (e != cudaSuccess) return e;
        if (per_sm < 1) return cudaErrorInvalidConfiguration;
        const uint64_t need = (a.nparticles + TPB - 1) / TPB;
        const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
        grid = (unsigned)(need < full ? need : full);
    } else {
        grid = (unsigned)((a.nparticles + TPB - 1) / TPB);
    }
    if (PT_MAP_PERSIST && REFILL && a.map) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(TPB);
        cfg.dynamicSmemBytes = dyn;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeAccessPolicyWindow;
        at[0].val.accessPolicyWindow.base_ptr = a.map;
        at[0].val.accessPolicyWindow.num_bytes = (size_t)a.nx * a.ny * a.nz * sizeof(uint32_t);
        at[0].val.accessPolicyWindow.hitRatio = 1.0f;
        at[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        size_t lim = 0;
        cudaDeviceGetLimit(&lim, cudaLimitPersistingL2CacheSize);
        if (lim < at[0].val.accessPolicyWindow.num_bytes)
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, at[0].val.accessPolicyWindow.num_bytes);
        cudaGetLastError();
        return cudaLaunchKernelEx(&cfg, k, a);
    }
    k<<<grid, TPB, dyn, st>>>(a);
    return cudaGetLastError();
}

template <int F, bool HALF>
static cudaError_t launch_f(const TrackArgs& a, bool simple, int num_sms, cudaStream_t st) {
    const bool out = a.o_nsteps || a.o_reason || a.o_end || a.o_paths;
    if (simple) return out ? launch_t<F, HALF, false, true>(a, num_sms, st) : launch_t<F, HALF, false, false>(a, num_sms, st);
    return out ? launch_t<F, HALF, true, true>(a, num_sms, st) : launch_t<F, HALF, true, false>(a, num_sms, st);
}

cudaError_t launch_track(const TrackArgs& a, int nfibres, bool half, bool simple, int num_sms,
                         cudaStream_t st) {
    switch (nfibres * 2 + (half ? 1 : 0)) {
        case 2: return launch_f<1, false>(a, simple, num_sms, st);
        case 3: return launch_f<1, true>(a, simple, num_sms, st);
        case 4: return launch_f<2, false>(a, simple, num_sms, st);
        case 5: return launch_f<2, true>(a, simple, num_sms, st);
        case 6: return launch_f<3, false>(a, simple, num_sms, st);
        case 7: return launch_f<3, true>(a, simple, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_repack(const void* dyads, const void* f, const uint8_t* mask, uint8_t* rec,
                          int64_t V, int S, int F, bool half, int rec_bytes,
                          unsigned long long* bad, cudaStream_t st) {
    const int64_t total = V * (int64_t)S;
    int64_t blocks = (total + 255) / 256;
    if (blocks > 148 * 64) blocks = 148 * 64;
    if (blocks < 1) blocks = 1;
    if (half)
        repack_kernel<true><<<(unsigned)blocks, 256, 0, st>>>(dyads, f, mask, rec, V, S, F, rec_bytes, bad);
    else
        repack_kernel<false><<<(unsigned)blocks, 256, 0, st>>>(dyads, f, mask, rec, V, S, F, rec_bytes, bad);
    return cudaGetLastError();
}

cudaError_t launch_map_sum(const uint32_t* map, int64_t V, unsigned long long* out, cudaStream_t st) {
    int64_t blocks = (V + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    map_sum_kernel<<<(unsigned)blocks, 256, 0, st>>>(map, V, out);
    return cudaGetLastError();
}

int gather_bench_blocks_per_sm(int rec_bytes) {
    int per_sm = 0;
    switch (rec_bytes) {
        case 8: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<8>, 256, 0); break;
        case 16: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<16>, 256, 0); break;
        case 32: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<32>, 256, 0); break;
        case 64: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<64>, 256, 0); break;
        default: break;
    }
    return per_sm;
}

cudaError_t launch_gather_bench(const uint8_t* buf, uint64_t nrec, int rec_bytes, uint32_t iters,
                                int blocks, uint32_t seed, uint32_t* sink, cudaStream_t st) {
    switch (rec_bytes) {
        case 8: gather_bench_kernel<8><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        case 16: gather_bench_kernel<16><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        case 32: gather_bench_kernel<32><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        case 64: gather_bench_kernel<64><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

}  // namespace pt
