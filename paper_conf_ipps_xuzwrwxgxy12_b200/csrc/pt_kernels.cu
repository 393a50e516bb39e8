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
#include <thrust/execution_policy.h>
#include <thrust/sort.h>

#include <cstdint>

#include "pt_device.cuh"
#include "pt_internal.h"

#ifndef PT_MIN_BLOCKS
#define PT_MIN_BLOCKS 1
#endif

namespace pt {

enum { kEndMask = 0, kEndCurv = 1, kEndMaxlen = 2 };

template <int F, bool HALF, bool REFILL>
__global__ void __launch_bounds__(kThreads, PT_MIN_BLOCKS) track_kernel(const __grid_constant__ TrackArgs a) {
    using R = Rec<F, HALF>;
    constexpr int RB = R::kBytes;
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t lt_mask = (1u << lane) - 1u;

    // ---- per-lane particle state
    bool alive = false;   // lane holds a particle in flight
    bool pend = false;    // a candidate step waits for the round-start gather (mask test)
    float qx = 0.f, qy = 0.f, qz = 0.f;   // committed position, centred coordinates (R10)
    float px = 0.f, py = 0.f, pz = 0.f;   // direction of the last (candidate) step
    float cqx = 0.f, cqy = 0.f, cqz = 0.f;  // pending candidate position
    uint32_t gvox = 0;    // voxel read by the round-start gather
    int n = 0;            // committed steps
    uint64_t pid = 0;     // global particle id = seed_id * P + j (RNG key, R16)
    uint64_t li = 0;      // particle index of this call = seed_index * P + j (outputs)
    uint32_t sign0 = 0;   // first step's sign bit
    uint32_t run_vox = 0, run_cnt = 0;  // run-length merge of consecutive visits
    R rv;                 // record of the current step
    uint4 W = make_uint4(0u, 0u, 0u, 0u);

    // ---- per-lane counters
    unsigned long long my_steps = 0, my_particles = 0, my_active = 0;
    unsigned long long rounds = 0;

    // ---- warp-uniform work-queue state
    uint64_t cseed = 0;
    uint32_t cnext = 0, cend = 0;
    bool exhausted = false;

    auto flush = [&]() {
        if (run_cnt) {
            atomicAdd(a.map + run_vox, run_cnt);  // no return value used -> RED
            run_cnt = 0;
        }
    };
    // SetEndPoint()
    auto finish = [&](int why) {
        if (a.o_nsteps) a.o_nsteps[li] = (uint16_t)n;
        if (a.o_reason) a.o_reason[li] = (uint8_t)why;
        if (a.o_end) {
            float* e = a.o_end + 3 * li;
            e[0] = __fadd_rn(qx, a.fcx);
            e[1] = __fadd_rn(qy, a.fcy);
            e[2] = __fadd_rn(qz, a.fcz);
        }
        if (a.map) flush();
        my_steps += (unsigned long long)n;
        my_particles += 1ull;
        alive = false;
        pend = false;
    };
    // commit a step: new position, one visit of the new voxel (R13)
    auto commit = [&](float x, float y, float z, uint32_t v) {
        qx = x;
        qy = y;
        qz = z;
        n += 1;
        if (a.map) {
            if (run_cnt != 0u && v == run_vox) {
                run_cnt += 1u;
            } else {
                flush();
                run_vox = v;
                run_cnt = 1u;
            }
        }
        if (a.o_paths && n < a.path_stride) {
            float* pp = a.o_paths + (li * (uint64_t)a.path_stride + (uint64_t)n) * 3u;
            pp[0] = __fadd_rn(qx, a.fcx);
            pp[1] = __fadd_rn(qy, a.fcy);
            pp[2] = __fadd_rn(qz, a.fcz);
        }
    };
    // GetStartPoint(): centred seed position, seed voxel (R10, R12)
    auto start = [&](uint64_t si, uint64_t j) {
        li = si * a.P + j;
        const uint64_t sid = a.seed_ids ? a.seed_ids[si] : si;
        pid = sid * a.P + j;
        qx = __fsub_rn(a.seeds[3 * si + 0], a.fcx);
        qy = __fsub_rn(a.seeds[3 * si + 1], a.fcy);
        qz = __fsub_rn(a.seeds[3 * si + 2], a.fcz);
        n = 0;
        pend = false;
        run_cnt = 0;
        alive = true;
        if (a.o_paths) {
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
            finish(kEndMask);
        }
    };

    if (!REFILL) {
        const uint64_t g = (uint64_t)blockIdx.x * kThreads + threadIdx.x;
        if (g < a.nparticles) {
            const uint64_t si = g / a.P;
            start(si, g - si * a.P);
        }
    }

    for (;;) {
        // ------------------------------------------------ lane refill (replaces the
        // paper's CPU Reduction()/segment relaunch)
        if (REFILL) {
            uint32_t need = __ballot_sync(kFull, !alive);
            while (need != 0u && !exhausted) {
                if (cnext == cend) {
                    unsigned long long c = 0;
                    if (lane == 0) c = atomicAdd(a.stats + kStatQueue, 1ull);
                    c = __shfl_sync(kFull, c, 0);
                    if (c >= a.total_chunks) {
                        exhausted = true;
                        break;
                    }
                    const uint64_t k = c / a.chunks_per_seed;
                    cnext = (uint32_t)(c - k * a.chunks_per_seed) * kChunk;
                    cseed = a.order ? (uint64_t)a.order[k] : k;
                    const uint64_t e = (uint64_t)cnext + kChunk;
                    cend = (uint32_t)(e < a.P ? e : a.P);
                }
                const uint32_t avail = cend - cnext;
                const uint32_t rank = __popc(need & lt_mask);
                if (!alive && rank < avail) start(cseed, (uint64_t)(cnext + rank));
                const uint32_t cnt = (uint32_t)__popc(need);
                cnext += cnt < avail ? cnt : avail;
                need = __ballot_sync(kFull, !alive);
            }
        }
        if (!__any_sync(kFull, alive)) break;
        rounds += 1ull;

        // ------------------------------------------------ round start: one Philox block,
        // gather of (pending candidate | seed) voxel = mask test + first step's record
        if (alive) {
            const uint32_t t0 = (uint32_t)n + (pend ? 1u : 0u);  // a multiple of 3
            W = philox4x32_10(make_uint4(t0 / 3u, (uint32_t)pid, (uint32_t)(pid >> 32), 0u),
                              a.key0, a.key1);
            ldg_record<RB>(a.rec + ((uint64_t)gvox * a.S + sample_of(W.x, a.S)) * RB, rv.w);
            if (rv.outside()) {
                finish(kEndMask);  // seed outside the mask (R12) or candidate rejected (R11)
            } else {
                if (pend) {
                    commit(cqx, cqy, cqz, gvox);
                    pend = false;
                }
                if (n == 0) sign0 = W.w >> 31;
            }
        }

        // ------------------------------------------------ three steps
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            my_active += alive ? 1ull : 0ull;
            if (alive) {
                if (n == a.max_steps) {
                    finish(kEndMaxlen);  // maximum number of steps (R14)
                } else {
                    float vx, vy, vz, fj;
                    bool go = true;
                    float sg;
                    if (n == 0) {
                        rv.fibre(0, vx, vy, vz, fj);  // R5, R6
                        sg = sign0 ? -1.f : 1.f;
                    } else {
                        // choose the fibre closest to the previous direction:
                        // eligible iff f_j > fib_thr (R7), strict >, lowest j wins (R8)
                        float bc = 0.f, best = -1.f;
                        rv.fibre(0, vx, vy, vz, fj);
                        {
                            const float c0 = __fadd_rn(__fadd_rn(__fmul_rn(vx, px), __fmul_rn(vy, py)),
                                                       __fmul_rn(vz, pz));
                            bc = c0;
                            if (fj > a.fib_thr) best = fabsf(c0);
                        }
#pragma unroll
                        for (int j = 1; j < F; ++j) {
                            float ux, uy, uz, fu;
                            rv.fibre(j, ux, uy, uz, fu);
                            const float cj = __fadd_rn(__fadd_rn(__fmul_rn(ux, px), __fmul_rn(uy, py)),
                                                       __fmul_rn(uz, pz));
                            if (fu > a.fib_thr && fabsf(cj) > best) {
                                best = fabsf(cj);
                                bc = cj;
                                vx = ux;
                                vy = uy;
                                vz = uz;
                            }
                        }
                        // maximum angle, measured by the dot product (R4)
                        if (!(fabsf(bc) > a.curv_thr)) {
                            finish(kEndCurv);
                            go = false;
                        }
                        sg = bc > 0.f ? 1.f : -1.f;  // keep the orientation (R9)
                    }
                    if (go) {
                        // StepToNextPoint(): q' = q + h * (sign * v), no FMA
                        const float dx = sg < 0.f ? -vx : vx;
                        const float dy = sg < 0.f ? -vy : vy;
                        const float dz = sg < 0.f ? -vz : vz;
                        px = dx;
                        py = dy;
                        pz = dz;
                        const float nqx = __fadd_rn(qx, __fmul_rn(a.step, dx));
                        const float nqy = __fadd_rn(qy, __fmul_rn(a.step, dy));
                        const float nqz = __fadd_rn(qz, __fmul_rn(a.step, dz));
                        const int ix = axis_index(nqx, a.cx), iy = axis_index(nqy, a.cy),
                                  iz = axis_index(nqz, a.cz);
                        if (!((unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny &&
                              (unsigned)iz < (unsigned)a.nz)) {
                            finish(kEndMask);  // left the volume (R11)
                        } else {
                            const uint32_t v =
                                ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
                            if (k < 2) {
                                const uint32_t w = (k == 0) ? W.y : W.z;
                                ldg_record<RB>(a.rec + ((uint64_t)v * a.S + sample_of(w, a.S)) * RB, rv.w);
                                if (rv.outside()) {
                                    finish(kEndMask);  // candidate outside the mask (R11)
                                } else {
                                    commit(nqx, nqy, nqz, v);
                                }
                            } else {
                                pend = true;  // next round's start gathers and tests it
                                cqx = nqx;
                                cqy = nqy;
                                cqz = nqz;
                                gvox = v;
                            }
                        }
                    }
                }
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
        atomicAdd(a.stats + kStatSteps, my_steps);
        atomicAdd(a.stats + kStatParticles, my_particles);
        atomicAdd(a.stats + kStatLaneActive, my_active);
        atomicAdd(a.stats + kStatLaneSlots, rounds * 3ull * 32ull);
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

__global__ void seed_keys_kernel(const float* __restrict__ seeds, uint64_t n, uint64_t* keys,
                                 uint32_t* perm) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t c[3];
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            const float x = seeds[3 * i + a];
            c[a] = x <= 0.f ? 0u : (x >= 1023.f ? 1023u : (uint32_t)x);
        }
        const uint64_t m = spread3(c[0]) | (spread3(c[1]) << 1) | (spread3(c[2]) << 2);
        keys[i] = (m << 32) | (uint64_t)(uint32_t)i;
        perm[i] = (uint32_t)i;
    }
}

cudaError_t launch_seed_order(const float* seeds, uint64_t nseeds, uint64_t* keys, uint32_t* perm,
                              cudaStream_t st) {
    if (nseeds == 0) return cudaSuccess;
    uint64_t blocks = (nseeds + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    seed_keys_kernel<<<(unsigned)blocks, 256, 0, st>>>(seeds, nseeds, keys, perm);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    thrust::sort_by_key(thrust::cuda::par.on(st), keys, keys + nseeds, perm);
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
template <int F, bool HALF, bool REFILL>
static cudaError_t launch_t(const TrackArgs& a, int num_sms, cudaStream_t st) {
    auto k = track_kernel<F, HALF, REFILL>;
    if (a.nparticles == 0) return cudaSuccess;
    unsigned grid;
    if (REFILL) {
        int per_sm = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kThreads, 0);
        if (e != cudaSuccess) return e;
        if (per_sm < 1) per_sm = 1;
        const uint64_t need = (a.nparticles + kThreads - 1) / kThreads;
        const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
        grid = (unsigned)(need < full ? need : full);
    } else {
        grid = (unsigned)((a.nparticles + kThreads - 1) / kThreads);
    }
    k<<<grid, kThreads, 0, st>>>(a);
    return cudaGetLastError();
}

template <int F, bool HALF>
static cudaError_t launch_f(const TrackArgs& a, bool simple, int num_sms, cudaStream_t st) {
    return simple ? launch_t<F, HALF, false>(a, num_sms, st) : launch_t<F, HALF, true>(a, num_sms, st);
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

template <int F, bool HALF, bool REFILL>
static int bps() {
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, track_kernel<F, HALF, REFILL>, kThreads, 0);
    return per_sm;
}

int track_blocks_per_sm(int nfibres, bool half, bool simple) {
    switch (nfibres * 4 + (half ? 2 : 0) + (simple ? 1 : 0)) {
        case 4: return bps<1, false, true>();
        case 5: return bps<1, false, false>();
        case 6: return bps<1, true, true>();
        case 7: return bps<1, true, false>();
        case 8: return bps<2, false, true>();
        case 9: return bps<2, false, false>();
        case 10: return bps<2, true, true>();
        case 11: return bps<2, true, false>();
        case 12: return bps<3, false, true>();
        case 13: return bps<3, false, false>();
        case 14: return bps<3, true, true>();
        case 15: return bps<3, true, false>();
        default: return 0;
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
