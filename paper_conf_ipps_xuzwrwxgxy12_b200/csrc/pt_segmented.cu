// pt_segmented.cu -- ablation (ii) of SURVEY §8(d): the paper's own load-balancing scheme
// on the B200, for comparison with the persistent lane-refill kernel.
//
// The paper (Sec. IV-B; Table IV) launches one thread per live
// streamline for a segment of NumIteration[i] steps, then compacts the live streamlines
// on the CPU ("Reduction()") and relaunches with the next interval, e.g. strategy B
// = {1, 2, 5, 10, 20, 50, 100, 200, 500}.  Here the segment kernel runs one thread per live
// particle for k steps on a state array, the compaction is a device stream compaction
// (cub::DeviceSelect::Flagged), and the host only reads the live count between segments
// (the paper's CPU<->GPU transfer shrinks to 4 bytes).  After the last interval of the
// schedule the last interval repeats until no particle is alive.  Results are identical to
// the main kernel (counter-based RNG keyed by (pid, n), R16); only the schedule differs.
#include <cuda_runtime.h>
#include <cub/device/device_select.cuh>

#include <cstdint>

#include "pt_device.cuh"
#include "pt_internal.h"

namespace pt {

namespace {

enum { kSMask = 0, kSCurv = 1, kSMaxlen = 2 };

// state of a batch particle (SoA in SegState)
__device__ __forceinline__ bool inside_volume(const TrackArgs& a, float qx, float qy, float qz, uint32_t& v) {
    const int ix = axis_index(qx, a.cx), iy = axis_index(qy, a.cy), iz = axis_index(qz, a.cz);
    const bool in = (unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz;
    v = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
    return in;
}

template <bool OUT>
__device__ __forceinline__ void seg_finish(const TrackArgs& a, const SegState& s, uint32_t i, int n, int why, float qx,
                                           float qy, float qz) {
    if (OUT) {
        const uint64_t li = s.li[i];
        PT_BOUND(a, li < a.out_n);
        if (a.o_nsteps) a.o_nsteps[li] = (uint16_t)n;
        if (a.o_reason) a.o_reason[li] = (uint8_t)why;
        if (a.o_end) {
            float* e = a.o_end + 3 * li;
            e[0] = __fadd_rn(qx, a.fcx);
            e[1] = __fadd_rn(qy, a.fcy);
            e[2] = __fadd_rn(qz, a.fcz);
        }
    }
}

// GetStartPoint() for batch particles [base, base + count)
template <bool OUT>
__global__ void seg_init_kernel(const __grid_constant__ TrackArgs a, SegState s, uint64_t base, uint32_t count) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += gridDim.x * blockDim.x) {
        const uint64_t g = base + i;                 // processing-order particle index
        const uint64_t k = g / a.P, j = g - k * a.P;
        PT_BOUND(a, k < a.nseeds);
        const uint64_t si = a.order ? a.order[k] : k;
        PT_BOUND(a, si < a.nseeds);
        uint64_t sid = a.seed_ids ? a.seed_ids[si] : si;
        if (sid > a.max_seed_id) {  // pid would overflow 64 bits: reported as PT_ERR_ARG
            atomicExch(a.stats + kStatBadId, 1ull);
            sid = 0;
        }
        s.li[i] = si * a.P + j;
        s.pid[i] = sid * a.P + j;
        const float qx = __fsub_rn(a.seeds[3 * si + 0], a.fcx);
        const float qy = __fsub_rn(a.seeds[3 * si + 1], a.fcy);
        const float qz = __fsub_rn(a.seeds[3 * si + 2], a.fcz);
        s.q[3 * i] = qx;
        s.q[3 * i + 1] = qy;
        s.q[3 * i + 2] = qz;
        s.p[3 * i] = s.p[3 * i + 1] = s.p[3 * i + 2] = 0.f;
        s.n[i] = 0u;
        uint32_t v;
        // non-finite seeds are outside (R12; a NaN would truncate into the volume)
        const bool fin = isfinite(qx) && isfinite(qy) && isfinite(qz);
        const bool inv = fin && inside_volume(a, qx, qy, qz, v);
        if (inv) PT_BOUND(a, v < a.V);
        const bool ok = inv && a.mask[v] != 0;
        s.vox[i] = v;
        s.live[i] = i;
        s.flag[i] = ok ? 1 : 0;
        if (!ok) {  // R12: seed outside the volume or the mask
            seg_finish<OUT>(a, s, i, 0, kSMask, qx, qy, qz);
            atomicAdd(a.stats + kStatParticles, 1ull);
        }
    }
}

// One segment: each live particle advances up to k steps (Alg. 1 inner loop).
template <int F, bool HALF, bool OUT>
__global__ void __launch_bounds__(256) seg_kernel(const __grid_constant__ TrackArgs a, SegState s, const uint32_t* live,
                                                  uint32_t nlive, uint32_t k) {
    using R = Rec<F, HALF>;
    constexpr int RB = R::kBytes;
    unsigned long long my_steps = 0, my_done = 0;
    uint32_t its = 0;  // loop iterations this lane ran (its SIMD occupancy)
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t < nlive) {
        const uint32_t i = live[t];
        float qx = s.q[3 * i], qy = s.q[3 * i + 1], qz = s.q[3 * i + 2];
        float px = s.p[3 * i], py = s.p[3 * i + 1], pz = s.p[3 * i + 2];
        int n = (int)s.n[i];
        uint32_t vox = s.vox[i];
        const uint64_t pid = s.pid[i];
        int why = -1;
        for (uint32_t it = 0; it < k; ++it) {
            its += 1;
            if (n == a.max_steps) {  // P:L116, R14
                why = kSMaxlen;
                break;
            }
            const uint4 W = philox4x32_10(make_uint4((uint32_t)n / 3u, (uint32_t)pid, (uint32_t)(pid >> 32), 0u), a.key0, a.key1);
            const int r3 = n % 3;
            const uint32_t wn = r3 == 0 ? W.x : (r3 == 1 ? W.y : W.z);
            const uint32_t smp = a.sample_mode ? (uint32_t)((s.li[i] % a.P) % a.S) : sample_of(wn, a.S);
            R rv;
            const uint32_t rvx = rec_vox_raster(vox, (uint32_t)a.nx, (uint32_t)a.ny, a.rb_log, a.rb_nbx, a.rb_nby, a.rb_off);
            PT_BOUND(a, (uint64_t)rvx * a.S + smp < a.rec_n && smp < a.S);
            ldg_record<RB>(a.rec + rec_slot(rvx, smp, a.S, a.rb_log) * RB, rv.w);
            float vx, vy, vz, f0;
            rv.fibre(0, vx, vy, vz, f0);
            bool neg;
            if (n == 0) {  // R5, R6
                neg = (W.w >> 31) != 0u;
            } else {       // P:L111, R7, R8, R4; R9
                float bc = __fadd_rn(__fadd_rn(__fmul_rn(vx, px), __fmul_rn(vy, py)), __fmul_rn(vz, pz));
                float best = f0 > a.fib_thr ? fabsf(bc) : -1.f;
#pragma unroll
                for (int j = 1; j < F; ++j) {
                    float ux, uy, uz, fu;
                    rv.fibre(j, ux, uy, uz, fu);
                    const float cj = __fadd_rn(__fadd_rn(__fmul_rn(ux, px), __fmul_rn(uy, py)), __fmul_rn(uz, pz));
                    if (fu > a.fib_thr && fabsf(cj) > best) {
                        best = fabsf(cj);
                        bc = cj;
                        vx = ux;
                        vy = uy;
                        vz = uz;
                    }
                }
                if (!(fabsf(bc) > a.curv_thr)) {
                    why = kSCurv;
                    break;
                }
                neg = !(bc > 0.f);
            }
            const float dx = neg ? -vx : vx, dy = neg ? -vy : vy, dz = neg ? -vz : vz;
            const float nqx = __fadd_rn(qx, __fmul_rn(a.step, dx));
            const float nqy = __fadd_rn(qy, __fmul_rn(a.step, dy));
            const float nqz = __fadd_rn(qz, __fmul_rn(a.step, dz));
            uint32_t v;
            const bool inv = inside_volume(a, nqx, nqy, nqz, v);
            if (inv) PT_BOUND(a, v < a.V);
            if (!inv || a.mask[v] == 0) {  // P:L177, R11
                why = kSMask;
                break;
            }
            qx = nqx;
            qy = nqy;
            qz = nqz;
            px = dx;
            py = dy;
            pz = dz;
            vox = v;
            n += 1;
            if (a.map) atomicAdd(a.map + map_cell(a, v), 1u);  // P:L109, R13 (plain global RED per step)
            my_steps += 1;
        }
        s.flag[t] = why >= 0 ? 0 : 1;  // by list position: the compaction's flags
        if (why >= 0) {
            seg_finish<OUT>(a, s, i, n, why, qx, qy, qz);
            my_done += 1;
        } else {
            s.q[3 * i] = qx;
            s.q[3 * i + 1] = qy;
            s.q[3 * i + 2] = qz;
            s.p[3 * i] = px;
            s.p[3 * i + 1] = py;
            s.p[3 * i + 2] = pz;
            s.n[i] = (uint32_t)n;
            s.vox[i] = vox;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        my_steps += __shfl_xor_sync(kFull, my_steps, o);
        my_done += __shfl_xor_sync(kFull, my_done, o);
    }
    // SIMD efficiency: a warp runs as long as its longest lane
    const uint32_t its_sum = __reduce_add_sync(kFull, its);
    const uint32_t its_max = __reduce_max_sync(kFull, its);
    if ((threadIdx.x & 31) == 0) {
        if (my_steps) atomicAdd(a.stats + kStatSteps, my_steps);
        if (my_done) atomicAdd(a.stats + kStatParticles, my_done);
        atomicAdd(a.stats + kStatLaneActive, (unsigned long long)its_sum);
        atomicAdd(a.stats + kStatLaneSlots, 32ull * its_max);
    }
}

template <int F, bool HALF, bool OUT>
cudaError_t seg_launch(const TrackArgs& a, const SegState& s, const uint32_t* live, uint32_t nlive, uint32_t k,
                       cudaStream_t st) {
    seg_kernel<F, HALF, OUT><<<(nlive + 255) / 256, 256, 0, st>>>(a, s, live, nlive, k);
    return cudaGetLastError();
}

template <bool OUT>
cudaError_t seg_dispatch(const TrackArgs& a, int F, bool half, const SegState& s, const uint32_t* live, uint32_t nlive,
                         uint32_t k, cudaStream_t st) {
    switch (F * 2 + (half ? 1 : 0)) {
        case 2: return seg_launch<1, false, OUT>(a, s, live, nlive, k, st);
        case 3: return seg_launch<1, true, OUT>(a, s, live, nlive, k, st);
        case 4: return seg_launch<2, false, OUT>(a, s, live, nlive, k, st);
        case 5: return seg_launch<2, true, OUT>(a, s, live, nlive, k, st);
        case 6: return seg_launch<3, false, OUT>(a, s, live, nlive, k, st);
        case 7: return seg_launch<3, true, OUT>(a, s, live, nlive, k, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace

size_t seg_select_temp_bytes(uint32_t n) {
    size_t bytes = 0;
    cub::DeviceSelect::Flagged(nullptr, bytes, (const uint32_t*)nullptr, (const uint8_t*)nullptr, (uint32_t*)nullptr,
                               (uint32_t*)nullptr, (int64_t)n);
    return bytes;
}

cudaError_t run_segmented(const TrackArgs& a, int F, bool half, const SegState& s, uint32_t batch,
                          const int32_t* schedule, int nsched, uint32_t* live_b, uint32_t* d_count, void* temp,
                          size_t temp_bytes, cudaStream_t st) {
    const bool out = a.o_nsteps || a.o_reason || a.o_end;
    for (uint64_t base = 0; base < a.nparticles; base += batch) {
        const uint32_t count = (uint32_t)((a.nparticles - base) < batch ? (a.nparticles - base) : batch);
        unsigned blocks = (count + 255) / 256;
        if (blocks > 148 * 64) blocks = 148 * 64;
        if (out) seg_init_kernel<true><<<blocks, 256, 0, st>>>(a, s, base, count);
        else seg_init_kernel<false><<<blocks, 256, 0, st>>>(a, s, base, count);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        // the seeds that are inside start live; compact once
        e = cub::DeviceSelect::Flagged(temp, temp_bytes, s.live, s.flag, live_b, d_count, (int64_t)count, st);
        if (e != cudaSuccess) return e;
        uint32_t nlive = 0;
        e = cudaMemcpyAsync(&nlive, d_count, sizeof nlive, cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) return e;
        uint32_t* cur = live_b;
        uint32_t* nxt = s.live;
        for (int seg = 0; nlive > 0; ++seg) {
            const uint32_t k = (uint32_t)schedule[seg < nsched ? seg : nsched - 1];
            e = out ? seg_dispatch<true>(a, F, half, s, cur, nlive, k, st)
                    : seg_dispatch<false>(a, F, half, s, cur, nlive, k, st);
            if (e != cudaSuccess) return e;
            // Reduction(): keep the live particles (device stream compaction)
            e = cub::DeviceSelect::Flagged(temp, temp_bytes, cur, s.flag, nxt, d_count, (int64_t)nlive, st);
            if (e != cudaSuccess) return e;
            e = cudaMemcpyAsync(&nlive, d_count, sizeof nlive, cudaMemcpyDeviceToHost, st);
            if (e == cudaSuccess) e = cudaStreamSynchronize(st);
            if (e != cudaSuccess) return e;
            uint32_t* tmp = cur;
            cur = nxt;
            nxt = tmp;
        }
    }
    return cudaSuccess;
}

}  // namespace pt
