// pt_variants.cu -- NEXT-3 FSL-fidelity variants of the particle stepper (sm_100a).
//
//   track_var_kernel : Algorithm 1's inner loop with the semantics of
//                      P:L98-121 plus the variants of DESIGN.md
//                        R22 bidirectional streamlines (two halves, the second starting
//                            against half 0's first direction),
//                        R23 probabilistic interpolation of the sampled voxel
//                            ("Interpolation()"),
//                        R24 random / f-weighted first fibre.
//
// Same work distribution as the main kernel (persistent CTAs, global claims, warp
// sub-chunks, ballot/popc lane refill; pt_claim.cuh) but one step per iteration instead of
// the main kernel's 6-step rounds, so a lane's RNG stream position, its half and the interpolation draws stay
// simple per-lane state.  Each step issues the next step's record gather (and, with
// interpolation, the 1-byte mask read of the candidate's nearest voxel) as soon as the
// candidate position is known, so one memory latency is exposed per step.  Without
// interpolation the record gather at the candidate's voxel doubles as its mask test (the
// sentinel records of the repack, R11) exactly as in the main kernel.
#include <cuda_runtime.h>

#include <cstdint>

#include "pt_claim.cuh"
#include "pt_device.cuh"
#include "pt_internal.h"

namespace pt {

namespace {

enum { kVMask = 0, kVCurv = 1, kVMaxlen = 2 };

// R23: per axis, the upper of the two voxels whose centres bracket q is taken with
// probability = its linear weight (t = q - 0.5, m = floor(t), fr = t - m, r = (w>>8) 2^-24).
__device__ __forceinline__ int interp_axis(float q, int c, uint32_t w) {
    const float t = __fsub_rn(q, 0.5f);
    const float m = floorf(t);
    const float fr = __fsub_rn(t, m);
    const float r = __fmul_rn(__uint2float_rn(w >> 8), 0x1p-24f);
    return c + __float2int_rz(m) + (r < fr ? 1 : 0);
}

template <int F, bool HALF>
struct VSlot {
    bool alive;             // particle (half) in flight
    bool pend;              // the candidate (or the seed, seedchk) awaits its mask test
    bool seedchk;           // the pending test is the seed voxel's (nothing to commit)
    bool have_d0;           // half 0 computed its first direction (R22)
    uint32_t half;          // 0, or 1 = the reverse half (R22)
    float qx, qy, qz;       // committed position, centred coordinates (R10)
    float px, py, pz;       // previous direction; the candidate's direction while pend
    float d0x, d0y, d0z;    // half 0's first-step direction (R22)
    uint32_t vox;           // nearest voxel of the committed position
    uint32_t cvox;          // nearest voxel of the candidate
    uint32_t rvox, crvox;   // their positions in the record volume (rec_vox)
    uint32_t s;             // sample index of the prefetched record
    uint32_t mb;            // prefetched mask byte of cvox / the seed voxel (interp)
    uint32_t wsign, winit;  // first step: stream 0 block 0 word 3 (R6); stream 2 word 3 (R24)
    int n;                  // committed steps of this half
    uint64_t pid;           // seed_id * P + j (RNG counter, R16)
    uint64_t li;            // seed index * P + j (output index before halves)
    uint32_t sfix;          // paper mode (NEXT-1): j mod S
    uint32_t sidx;          // seed index of this call
    uint32_t run_vox, run_cnt;
    int why;                // >= 0: ended with this reason, outputs pending
    uint64_t tmask;         // NEXT-2 targets entered (both halves)
    Rec<F, HALF> rv;        // prefetched record of the next step
};

template <int F, bool HALF, bool OUT>
__global__ void __launch_bounds__(kVarThreads, 1) track_var_kernel(const __grid_constant__ TrackArgs a) {
    using R = Rec<F, HALF>;
    constexpr int RB = R::kBytes;
    __shared__ uint32_t s_q[kVarThreads / 32][3];
    __shared__ unsigned long long s_work;
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t wib = threadIdx.x >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    uint32_t* const map = a.map;
    const uint32_t H = a.bidir ? 2u : 1u;
    if (threadIdx.x == 0) s_work = kNoChunk << 24;
    if (lane == 0) {
        s_q[wib][0] = 0u;
        s_q[wib][1] = 0u;
        s_q[wib][2] = 0u;
    }
    __syncthreads();

    VSlot<F, HALF> x;
    x.alive = x.pend = x.seedchk = x.have_d0 = false;
    x.half = 0u;
    x.qx = x.qy = x.qz = x.px = x.py = x.pz = x.d0x = x.d0y = x.d0z = 0.f;
    x.vox = x.cvox = x.rvox = x.crvox = x.s = x.mb = x.wsign = x.winit = 0u;
    x.n = 0;
    x.pid = x.li = 0ull;
    x.sfix = x.sidx = x.run_vox = x.run_cnt = 0u;
    x.why = -1;
    x.tmask = 0ull;
#pragma unroll
    for (int k = 0; k < R::kWords; ++k) x.rv.w[k] = 0u;

    uint32_t my_steps = 0, my_particles = 0, my_active = 0, iters = 0;
    bool exhausted = false;  // warp-uniform

    auto nearest = [&](float qx, float qy, float qz, uint32_t& v, uint32_t& rv) -> bool {
        const int ix = axis_index(qx, a.cx), iy = axis_index(qy, a.cy), iz = axis_index(qz, a.cz);
        const bool in = (unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz;
        v = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
        rv = rec_vox(ix, iy, iz, a.rb_log, a.rb_nbx, a.rb_nby);
        return in;
    };
    // Issue the loads step n will need at position (qx,qy,qz) with nearest voxel nv:
    // the sample index (R1/R16: stream = half, block n/3, word n%3), the interpolated voxel
    // (R23: stream 2 + half, block n), the record gather, and the candidate's mask byte.
    auto prefetch = [&](float qx, float qy, float qz, uint32_t nv, uint32_t nrv, int n) {
        const uint32_t lo = (uint32_t)x.pid, hi = (uint32_t)(x.pid >> 32);
        const uint4 W = philox4x32_10(make_uint4((uint32_t)n / 3u, lo, hi, x.half), a.key0, a.key1);
        const int r3 = n % 3;
        const uint32_t wn = r3 == 0 ? W.x : (r3 == 1 ? W.y : W.z);
        x.s = a.sample_mode ? x.sfix : sample_of(wn, a.S);
        const bool first = n == 0 && x.half == 0u;
        if (first) x.wsign = W.w;
        uint32_t ur = nrv;
        if (a.interp || (first && a.init_mode)) {
            const uint4 I = philox4x32_10(make_uint4((uint32_t)n, lo, hi, 2u + x.half), a.key0, a.key1);
            if (first) x.winit = I.w;
            if (a.interp) {
                const int ix = interp_axis(qx, a.cx, I.x), iy = interp_axis(qy, a.cy, I.y), iz = interp_axis(qz, a.cz, I.z);
                if ((unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz)
                    ur = rec_vox(ix, iy, iz, a.rb_log, a.rb_nbx, a.rb_nby);
            }
        }
        ldg_record<RB>(a.rec + ((uint64_t)ur * a.S + x.s) * RB, x.rv.w);
        if (a.interp) x.mb = __ldg(a.mask + nv);
    };
    // GetStartPoint() of the current half: centred seed position, RNG stream,
    // first prefetch.  Returns false if the seed is outside the volume (R12).
    auto begin_half = [&]() -> bool {
        x.qx = __fsub_rn(a.seeds[3 * x.sidx + 0], a.fcx);
        x.qy = __fsub_rn(a.seeds[3 * x.sidx + 1], a.fcy);
        x.qz = __fsub_rn(a.seeds[3 * x.sidx + 2], a.fcz);
        x.n = 0;
        x.run_cnt = 0u;
        if (OUT && a.o_paths) {
            float* pp = a.o_paths + (x.li * H + x.half) * (uint64_t)a.path_stride * 3u;
            pp[0] = __fadd_rn(x.qx, a.fcx);
            pp[1] = __fadd_rn(x.qy, a.fcy);
            pp[2] = __fadd_rn(x.qz, a.fcz);
        }
        if (!nearest(x.qx, x.qy, x.qz, x.vox, x.rvox)) return false;
        x.cvox = x.vox;
        x.crvox = x.rvox;
        prefetch(x.qx, x.qy, x.qz, x.vox, x.rvox, 0);
        return true;
    };
    auto write_outputs = [&]() {
        if (OUT && (a.o_nsteps || a.o_reason || a.o_end)) {
            const uint64_t e = x.li * H + x.half;
            if (a.o_nsteps) a.o_nsteps[e] = (uint16_t)x.n;
            if (a.o_reason) a.o_reason[e] = (uint8_t)x.why;
            if (a.o_end) {
                float* o = a.o_end + 3 * e;
                o[0] = __fadd_rn(x.qx, a.fcx);
                o[1] = __fadd_rn(x.qy, a.fcy);
                o[2] = __fadd_rn(x.qz, a.fcz);
            }
        }
        if (map && x.run_cnt) atomicAdd(map + x.run_vox, x.run_cnt);
        x.run_cnt = 0u;
        my_steps += (uint32_t)x.n;
    };
    // SetEndPoint() of a finished half; half 0 of a bidirectional particle
    // restarts as half 1 (R22).
    auto finish = [&]() {
        write_outputs();
        if (H == 2u && x.half == 0u) {
            x.half = 1u;
            x.why = -1;
            x.px = -x.d0x;
            x.py = -x.d0y;
            x.pz = -x.d0z;
            const bool ok = begin_half() && x.have_d0;
            if (ok) {
                x.alive = true;
                x.pend = false;  // the seed voxel passed its test in half 0
                return;
            }
            x.n = 0;  // seed outside: half 1 is empty too (R12)
            x.why = kVMask;
            write_outputs();
        }
        if (OUT && a.conn) {  // NEXT-2: one count per target the streamline entered
            uint64_t m = x.tmask;
            while (m) {
                const int t = __ffsll((long long)m) - 1;
                atomicAdd(a.conn + (uint64_t)x.sidx * a.ntargets + (uint32_t)t, 1u);
                m &= m - 1ull;
            }
            x.tmask = 0ull;
        }
        my_particles += 1u;
        x.why = -1;
    };
    auto start = [&](uint64_t si, uint64_t j) {
        const uint64_t sid = a.seed_ids ? a.seed_ids[si] : si;
        x.pid = sid * a.P + j;
        x.li = si * a.P + j;
        x.sidx = (uint32_t)si;
        x.sfix = (uint32_t)(j % a.S);
        x.half = 0u;
        x.have_d0 = false;
        x.tmask = 0ull;
        x.px = x.py = x.pz = 0.f;
        x.why = -1;
        if (begin_half()) {
            x.alive = true;
            x.pend = true;
            x.seedchk = true;
        } else {
            x.alive = false;
            x.pend = false;
            x.why = kVMask;
            finish();  // may restart as half 1 (which then ends at once)
        }
    };

    for (;;) {
        if (x.why >= 0) finish();

        // ------------------------------------------------ lane refill (pt_claim.cuh)
        if (__any_sync(kFull, !x.alive) && !exhausted) {
            uint32_t cseed = s_q[wib][0], cnext = s_q[wib][1], cend = s_q[wib][2];
            uint32_t need = __ballot_sync(kFull, !x.alive);
            while (need != 0u && !exhausted) {
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
                if (!x.alive && rank < avail) start(cseed, (uint64_t)(cnext + rank));
                const uint32_t cnt = (uint32_t)__popc(need);
                cnext += cnt < avail ? cnt : avail;
                need = __ballot_sync(kFull, !x.alive);
            }
            __syncwarp();
            if (lane == 0) {
                s_q[wib][0] = cseed;
                s_q[wib][1] = cnext;
                s_q[wib][2] = cend;
            }
            __syncwarp();
        }
        if (!__any_sync(kFull, x.alive)) break;
        iters += 1u;
        my_active += x.alive ? 1u : 0u;
        if (!x.alive) continue;

        // ---- A: the pending test (R11: candidate; R12: seed) and the commit
        if (x.pend) {
            const bool inside = a.interp ? x.mb != 0u : !x.rv.outside();
            if (!inside) {
                x.alive = false;
                x.pend = false;
                x.why = kVMask;
                continue;
            }
            if (!x.seedchk) {
                // commit (R13): q' recomputed bit-identically from (q, d)
                x.qx = __fadd_rn(x.qx, __fmul_rn(a.step, x.px));
                x.qy = __fadd_rn(x.qy, __fmul_rn(a.step, x.py));
                x.qz = __fadd_rn(x.qz, __fmul_rn(a.step, x.pz));
                x.vox = x.cvox;
                x.rvox = x.crvox;
                x.n += 1;
                if (map) {
                    if (x.vox != x.run_vox || x.run_cnt == 0u) {
                        if (x.run_cnt) atomicAdd(map + x.run_vox, x.run_cnt);
                        x.run_vox = x.vox;
                        x.run_cnt = 1u;
                    } else {
                        x.run_cnt += 1u;
                    }
                }
                if (OUT && a.conn) {
                    const uint32_t lbl = __ldg(a.labels + x.vox);
                    x.tmask |= lbl ? (1ull << (lbl - 1u)) : 0ull;
                }
                if (OUT && a.o_paths && x.n < a.path_stride) {
                    float* pp = a.o_paths + ((x.li * H + x.half) * (uint64_t)a.path_stride + (uint64_t)x.n) * 3u;
                    pp[0] = __fadd_rn(x.qx, a.fcx);
                    pp[1] = __fadd_rn(x.qy, a.fcy);
                    pp[2] = __fadd_rn(x.qz, a.fcz);
                }
            }
            x.pend = false;
            x.seedchk = false;
        }

        // ---- maximum number of steps (R14), checked first
        if (x.n == a.max_steps) {
            x.alive = false;
            x.why = kVMaxlen;
            continue;
        }

        // ---- B: the interpolated voxel was outside the mask => nearest voxel (R23)
        if (a.interp && x.rv.outside()) ldg_record<RB>(a.rec + ((uint64_t)x.rvox * a.S + x.s) * RB, x.rv.w);

        // ---- C: fibre choice, curvature, step
        const bool first = x.n == 0 && x.half == 0u;
        float vx, vy, vz, bc;
        bool neg;
        if (first) {
            // R5 / R24: the first fibre; R6: sign from stream 0 block 0 word 3
            int js = 0;
            if (a.init_mode) {
                int el[3];
                int ne = 0;
                float fv[3];
#pragma unroll
                for (int j = 0; j < F; ++j) {
                    float ux, uy, uz;
                    x.rv.fibre(j, ux, uy, uz, fv[j]);
                    if (fv[j] > a.fib_thr) el[ne++] = j;
                }
                if (ne > 0) {
                    if (a.init_mode == 1u) {
                        js = el[__umulhi(x.winit, (uint32_t)ne)];
                    } else {
                        float tot = 0.f;
                        for (int k = 0; k < ne; ++k) tot = __fadd_rn(tot, fv[el[k]]);
                        const float r = __fmul_rn(__fmul_rn(__uint2float_rn(x.winit >> 8), 0x1p-24f), tot);
                        float cum = 0.f;
                        js = el[ne - 1];
                        for (int k = 0; k < ne; ++k) {
                            cum = __fadd_rn(cum, fv[el[k]]);
                            if (r < cum) {
                                js = el[k];
                                break;
                            }
                        }
                    }
                }
            }
            float fj;
            x.rv.fibre(0, vx, vy, vz, fj);
#pragma unroll
            for (int j = 1; j < F; ++j)
                if (j == js) x.rv.fibre(j, vx, vy, vz, fj);
            bc = 0.f;
            neg = (x.wsign >> 31) != 0u;
        } else {
            // the fibre closest to the previous direction (R7 eligibility, R8 ties)
            float f0;
            x.rv.fibre(0, vx, vy, vz, f0);
            bc = __fadd_rn(__fadd_rn(__fmul_rn(vx, x.px), __fmul_rn(vy, x.py)), __fmul_rn(vz, x.pz));
            float best = f0 > a.fib_thr ? fabsf(bc) : -1.f;
#pragma unroll
            for (int j = 1; j < F; ++j) {
                float ux, uy, uz, fu;
                x.rv.fibre(j, ux, uy, uz, fu);
                const float cj = __fadd_rn(__fadd_rn(__fmul_rn(ux, x.px), __fmul_rn(uy, x.py)), __fmul_rn(uz, x.pz));
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
                x.alive = false;
                x.why = kVCurv;
                continue;
            }
            neg = !(bc > 0.f);  // keep the orientation (R9)
        }
        const float dx = neg ? -vx : vx, dy = neg ? -vy : vy, dz = neg ? -vz : vz;
        if (first) {  // R22: d0
            x.d0x = dx;
            x.d0y = dy;
            x.d0z = dz;
            x.have_d0 = true;
        }
        // StepToNextPoint(): q' = q + h d, no FMA
        const float nqx = __fadd_rn(x.qx, __fmul_rn(a.step, dx));
        const float nqy = __fadd_rn(x.qy, __fmul_rn(a.step, dy));
        const float nqz = __fadd_rn(x.qz, __fmul_rn(a.step, dz));
        uint32_t v, rv;
        if (!nearest(nqx, nqy, nqz, v, rv)) {  // outside the volume (R11)
            x.alive = false;
            x.why = kVMask;
            continue;
        }
        x.px = dx;
        x.py = dy;
        x.pz = dz;
        x.cvox = v;
        x.crvox = rv;
        x.pend = true;
        prefetch(nqx, nqy, nqz, v, rv, x.n + 1);
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
        atomicAdd(a.stats + kStatLaneSlots, (unsigned long long)iters * 32ull);
    }
}

template <int F, bool HALF, bool OUT>
cudaError_t launch_v(const TrackArgs& a, int num_sms, cudaStream_t st) {
    auto k = track_var_kernel<F, HALF, OUT>;
    if (a.nparticles == 0) return cudaSuccess;
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kVarThreads, 0);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    const uint64_t need = (a.nparticles + kVarThreads - 1) / kVarThreads;
    const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
    k<<<(unsigned)(need < full ? need : full), kVarThreads, 0, st>>>(a);
    return cudaGetLastError();
}

template <int F, bool HALF>
cudaError_t launch_vf(const TrackArgs& a, int num_sms, cudaStream_t st) {
    const bool out = a.o_nsteps || a.o_reason || a.o_end || a.o_paths || a.conn;
    return out ? launch_v<F, HALF, true>(a, num_sms, st) : launch_v<F, HALF, false>(a, num_sms, st);
}

}  // namespace

cudaError_t launch_track_var(const TrackArgs& a, int nfibres, bool half, int num_sms, cudaStream_t st) {
    switch (nfibres * 2 + (half ? 1 : 0)) {
        case 2: return launch_vf<1, false>(a, num_sms, st);
        case 3: return launch_vf<1, true>(a, num_sms, st);
        case 4: return launch_vf<2, false>(a, num_sms, st);
        case 5: return launch_vf<2, true>(a, num_sms, st);
        case 6: return launch_vf<3, false>(a, num_sms, st);
        case 7: return launch_vf<3, true>(a, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace pt
