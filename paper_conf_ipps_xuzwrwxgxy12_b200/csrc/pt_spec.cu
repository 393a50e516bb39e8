// pt_spec.cu -- the default tracking kernel: persistent warps with lane refill (as in
// track_kernel, pt_kernels.cu) plus a SPECULATIVE second gather per lane and iteration.
//
// Why: the stepping chain of one particle is a dependent sequence of random gathers
// (Alg. 1's inner loop: the record of step t+1 lives in the voxel step t
// reaches).  With one gather in flight per lane, the kernel is bound by the DRAM latency
// tail of every warp-step, not by bandwidth.  Because the RNG is
// counter-based (R16), the SAMPLE index of step t+2 is known before step t+1 is taken;
// only its VOXEL is not.  Tracts are smooth (consecutive sample directions differ by the
// dispersion of one voxel's samples, and the step is 0.5 voxel), so the voxel the next
// candidate reaches is, most of the time, the one reached by extrapolating the current
// direction.  Each iteration therefore issues, back to back, the gather the particle
// needs (the pending candidate's record = its mask test + the next step's record, as in
// track_kernel) and the gather of the record of the step after it at the extrapolated
// voxel.  When the candidate that the next step actually produces lands in that voxel,
// the lane takes a second step in the same iteration without waiting; otherwise the
// speculative record is dropped.  Results are unchanged by construction: a speculative
// record is used only when it is exactly the record (voxel, sample) the sequential
// algorithm reads (C-ALG), so every parity test also covers this kernel.
//
// Iteration of one lane (alive particle, committed position q, n steps, candidate
// c = q + h p pending at voxel gvox, records R = rec[gvox][s_{n+1}] and
// S = rec[svox][s_{n+2}] landed):
//   A  R.outside -> end MASK (R11), else commit c (n+1)            [fresh seed: R12 test only]
//   B  step with R: fibre choice, curvature, q' = q + h d, voxel v1 (maxlen, curv, bounds)
//   C  if v1 == svox: S.outside -> end MASK, else commit, step with S -> candidate v2
//   D  gather R <- rec[v][s_t], S <- rec[lookup(c + h p)][s_{t+1}] (t = n + pending)
// Philox blocks (R16: block b gives steps 3b..3b+2) are cached as a pair (block ba, and
// block ba+1 once needed), so a lane computes at most one block per iteration.
#include <cuda_runtime.h>

#include <cstdint>

#include "pt_claim.cuh"
#include "pt_device.cuh"
#include "pt_internal.h"

#ifndef PT_SPEC_THREADS
#define PT_SPEC_THREADS 768
#endif
#ifndef PT_SPEC_REFILL_MIN
#define PT_SPEC_REFILL_MIN 2
#endif

namespace pt {

namespace {

enum { kEndMask = 0, kEndCurv = 1, kEndMaxlen = 2 };
constexpr int kSpecThreads = PT_SPEC_THREADS;

template <int F, bool HALF, bool OUT, int BL>
__global__ void __launch_bounds__(kSpecThreads, 1) track_spec_kernel(const __grid_constant__ TrackArgs a) {
    using R = Rec<F, HALF>;
    constexpr int RB = R::kBytes;
    constexpr int TPB = kSpecThreads;
    __shared__ unsigned long long s_li[OUT ? TPB : 1];  // particle index (outputs)
    __shared__ uint32_t s_q[TPB / 32][3];               // per-warp sub-chunk
    __shared__ unsigned long long s_work;               // CTA claim + tickets
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t wib = threadIdx.x >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const bool has_map = a.map != nullptr;
    uint32_t* const map = has_map ? a.map + (size_t)(blockIdx.x % a.map_copies) * ((size_t)a.nx * a.ny * a.nz)
                                  : nullptr;
    if (threadIdx.x == 0) s_work = kNoChunk << 24;
    if (lane == 0) {
        s_q[wib][0] = 0u;
        s_q[wib][1] = 0u;
        s_q[wib][2] = 0u;
    }
    __syncthreads();

    // ---- particle state of this lane
    bool alive = false, pend = false;
    float qx = 0.f, qy = 0.f, qz = 0.f;  // committed position, centred coordinates (R10)
    float px = 0.f, py = 0.f, pz = 0.f;  // direction of the pending candidate / last step
    uint32_t gvox = 0u, grv = 0u;        // candidate (or seed) voxel: raster / record position
    uint32_t svox = 0xFFFFFFFFu;         // voxel of the speculative record (none: ~0)
    int n = 0;
    uint64_t pid = 0ull;
    uint32_t run_vox = 0u, run_cnt = 0u;
    uint32_t sfix = 0u;
    int why = -1;
    uint4 Wa = make_uint4(0u, 0u, 0u, 0u), Wb = Wa;  // Philox blocks ba and ba + 1
    uint32_t ba = 0xFFFFFFFFu;
    bool hb = false;
    R rv, sv;
#pragma unroll
    for (int k = 0; k < R::kWords; ++k) rv.w[k] = sv.w[k] = 0u;
    uint64_t tmask = 0ull;
    uint32_t sidx = 0u;

    uint32_t my_steps = 0, my_particles = 0, my_active = 0, iters = 0, my_spec = 0;
    bool exhausted = false;  // warp-uniform

    auto recv = [&](int ix, int iy, int iz, uint32_t v) -> uint32_t {
        if (BL == 0) return v;
        constexpr uint32_t m = (1u << BL) - 1u;
        const uint32_t x = (uint32_t)ix, y = (uint32_t)iy, z = (uint32_t)iz;
        const uint32_t br = ((z >> BL) * a.rb_nby + (y >> BL)) * a.rb_nbx + (x >> BL);
        return (br << (3 * BL)) | ((z & m) << (2 * BL)) | ((y & m) << BL) | (x & m);
    };
    auto word = [&](uint32_t t) -> uint32_t {  // Philox word of step t (R16)
        const uint4& W = (t / 3u == ba) ? Wa : Wb;
        const uint32_t r = t - (t / 3u) * 3u;
        return r == 0u ? W.x : (r == 1u ? W.y : W.z);
    };
    // SetEndPoint(): outputs and the count flush of an ended particle
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
        if (has_map && run_cnt) atomicAdd(map + run_vox, run_cnt);
        run_cnt = 0;
        if (OUT && a.conn) {  // NEXT-2: one count per target the streamline entered
            uint64_t m = tmask;
            while (m) {
                const int t = __ffsll((long long)m) - 1;
                atomicAdd(a.conn + (uint64_t)sidx * a.ntargets + (uint32_t)t, 1u);
                m &= m - 1ull;
            }
            tmask = 0ull;
        }
        my_steps += (uint32_t)n;
        my_particles += 1u;
        why = -1;
    };
    // commit (if c) the step to (nx_, ny_, nz_) in voxel v: one visit of v (R13),
    // consecutive visits of a voxel merged into one RED (run length)
    auto commit_if = [&](bool c, float nx_, float ny_, float nz_, uint32_t v) {
        qx = c ? nx_ : qx;
        qy = c ? ny_ : qy;
        qz = c ? nz_ : qz;
        n += c ? 1 : 0;
        if (has_map) {
            const bool change = v != run_vox;
            red_add_if(c && change && run_cnt != 0u, map + run_vox, run_cnt);
            run_cnt = c ? (change ? 1u : run_cnt + 1u) : run_cnt;
            run_vox = c ? v : run_vox;
        }
        if (OUT && a.conn && c) {
            const uint32_t lbl = __ldg(a.labels + v);
            tmask |= lbl ? (1ull << (lbl - 1u)) : 0ull;
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
        sfix = a.sample_mode ? (uint32_t)(j % a.S) : 0u;
        tmask = 0ull;
        sidx = (uint32_t)si;
        qx = __fsub_rn(a.seeds[3 * si + 0], a.fcx);
        qy = __fsub_rn(a.seeds[3 * si + 1], a.fcy);
        qz = __fsub_rn(a.seeds[3 * si + 2], a.fcz);
        n = 0;
        pend = false;
        run_cnt = 0;
        alive = true;
        ba = 0xFFFFFFFFu;
        hb = false;
        if (OUT && a.o_paths) {
            float* pp = a.o_paths + li * (uint64_t)a.path_stride * 3u;
            pp[0] = __fadd_rn(qx, a.fcx);
            pp[1] = __fadd_rn(qy, a.fcy);
            pp[2] = __fadd_rn(qz, a.fcz);
        }
        const int ix = axis_index(qx, a.cx), iy = axis_index(qy, a.cy), iz = axis_index(qz, a.cz);
        if ((unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz) {
            gvox = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
            grv = recv(ix, iy, iz, gvox);
        } else {
            why = kEndMask;  // seed outside the volume (R12)
            alive = false;
            finish();
        }
    };
    // one step of Alg. 1's inner loop with record r; returns the candidate
    // (position, voxel, in-volume flag); ends the particle on maxlen / angle / volume
    auto step = [&](const R& r, bool live, float& cx_, float& cy_, float& cz_, uint32_t& v, int& ix, int& iy,
                    int& iz) -> bool {
        const bool first = n == 0;
        float vx, vy, vz, f0;
        r.fibre(0, vx, vy, vz, f0);
        float bc = __fadd_rn(__fadd_rn(__fmul_rn(vx, px), __fmul_rn(vy, py)), __fmul_rn(vz, pz));
        float best = f0 > a.fib_thr ? fabsf(bc) : -1.f;
#pragma unroll
        for (int j = 1; j < F; ++j) {  // closest eligible fibre (R7, R8), fibre 0 first (R5)
            float ux, uy, uz, fu;
            r.fibre(j, ux, uy, uz, fu);
            const float cj = __fadd_rn(__fadd_rn(__fmul_rn(ux, px), __fmul_rn(uy, py)), __fmul_rn(uz, pz));
            const bool pick = !first && fu > a.fib_thr && fabsf(cj) > best;
            best = pick ? fabsf(cj) : best;
            bc = pick ? cj : bc;
            vx = pick ? ux : vx;
            vy = pick ? uy : vy;
            vz = pick ? uz : vz;
        }
        // maximum angle by the dot product (R4); sign (R6, R9)
        const bool curv_ok = first || fabsf(bc) > a.curv_thr;
        const bool neg = first ? (Wa.w >> 31) != 0u : !(bc > 0.f);
        const float dx = neg ? -vx : vx, dy = neg ? -vy : vy, dz = neg ? -vz : vz;
        // StepToNextPoint(), no FMA
        cx_ = __fadd_rn(qx, __fmul_rn(a.step, dx));
        cy_ = __fadd_rn(qy, __fmul_rn(a.step, dy));
        cz_ = __fadd_rn(qz, __fmul_rn(a.step, dz));
        ix = axis_index(cx_, a.cx);
        iy = axis_index(cy_, a.cy);
        iz = axis_index(cz_, a.cz);
        const bool inb = (unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz;
        v = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
        // stop criteria in order: maximum steps (R14), angle, volume (R11)
        const bool maxed = n == a.max_steps;
        const bool go = live && !maxed && curv_ok && inb;
        why = (live && !go) ? (maxed ? kEndMaxlen : (!curv_ok ? kEndCurv : kEndMask)) : why;
        px = go ? dx : px;
        py = go ? dy : py;
        pz = go ? dz : pz;
        return go;
    };

    for (;;) {
        if (why >= 0) finish();  // particle that ended in the last iteration

        // ------------------------------------------------ lane refill (replaces the paper's
        // CPU Reduction()/segment relaunch)
        {
            const uint32_t nfree = (uint32_t)__popc(__ballot_sync(kFull, !alive));
            if (!exhausted && nfree != 0u && (nfree >= (uint32_t)PT_SPEC_REFILL_MIN || nfree == 32u)) {
                uint32_t cseed = s_q[wib][0], cnext = s_q[wib][1], cend = s_q[wib][2];
                uint32_t need = __ballot_sync(kFull, !alive);
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
        iters += 1u;
        my_active += alive ? 1u : 0u;

        // ------------------------------------------------ D: gathers of this iteration
        // t = index of the step the pending candidate's record serves (R16)
        const uint32_t t = (uint32_t)n + (pend ? 1u : 0u);
        const uint32_t bR = t / 3u;
        // the speculative record (pending candidate extrapolated by one more step)
        const float ex = __fadd_rn(__fadd_rn(qx, __fmul_rn(a.step, px)), __fmul_rn(a.step, px));
        const float ey = __fadd_rn(__fadd_rn(qy, __fmul_rn(a.step, py)), __fmul_rn(a.step, py));
        const float ez = __fadd_rn(__fadd_rn(qz, __fmul_rn(a.step, pz)), __fmul_rn(a.step, pz));
        const int sx = axis_index(ex, a.cx), sy = axis_index(ey, a.cy), sz = axis_index(ez, a.cz);
        const bool sinb = (unsigned)sx < (unsigned)a.nx && (unsigned)sy < (unsigned)a.ny && (unsigned)sz < (unsigned)a.nz;
        // Philox: block bR into Wa (shifted from Wb when it is already there), else block
        // bR + 1 into Wb when the speculative draw needs it: at most one block per lane
        const bool shift = alive && bR != ba && bR == ba + 1u && hb;
        if (shift) {
            Wa = Wb;
            ba = bR;
            hb = false;
        }
        // (paper mode, NEXT-1: the sample is fixed per particle; only block 0 is drawn)
        const bool needA = alive && bR != ba && !(a.sample_mode && ba == 0u);
        const bool wantS = alive && pend && sinb;
        const bool needB = !needA && wantS && !a.sample_mode && (t + 1u) / 3u != ba && !hb;
        const bool specok = wantS && (!needA || a.sample_mode);
        if (needA || needB) {
            const uint4 W = philox4x32_10(make_uint4(needA ? (a.sample_mode ? 0u : bR) : ba + 1u, (uint32_t)pid,
                                                     (uint32_t)(pid >> 32), 0u),
                                          a.key0, a.key1);
            Wa = needA ? W : Wa;
            ba = needA ? (a.sample_mode ? 0u : bR) : ba;
            Wb = needB ? W : Wb;
            hb = needB ? true : (needA ? false : hb);
        }
        const uint32_t s0 = a.sample_mode ? sfix : sample_of(word(t), a.S);
        ldg_record_if<RB>(alive, a.rec + ((uint64_t)(BL == 0 ? gvox : grv) * a.S + s0) * RB, rv.w);
        const uint32_t sv_raster = ((uint32_t)sz * (uint32_t)a.ny + (uint32_t)sy) * (uint32_t)a.nx + (uint32_t)sx;
        const uint32_t s1 = a.sample_mode ? sfix : sample_of(word(t + 1u), a.S);
        ldg_record_if<RB>(specok, a.rec + ((uint64_t)recv(sx, sy, sz, sv_raster) * a.S + s1) * RB, sv.w);
        svox = specok ? sv_raster : 0xFFFFFFFFu;

        // ------------------------------------------------ A: mask test of the candidate
        // (or of the seed, R12) = the gathered record's sentinel (R11); commit
        {
            const bool outside = alive && rv.outside();
            why = outside ? kEndMask : why;
            alive = alive && !outside;
            commit_if(pend && !outside, __fadd_rn(qx, __fmul_rn(a.step, px)), __fadd_rn(qy, __fmul_rn(a.step, py)),
                      __fadd_rn(qz, __fmul_rn(a.step, pz)), gvox);
            pend = false;
        }
        // ------------------------------------------------ B: step with R
        float c1x, c1y, c1z;
        uint32_t v1;
        int i1x, i1y, i1z;
        const bool go1 = step(rv, alive, c1x, c1y, c1z, v1, i1x, i1y, i1z);
        // ------------------------------------------------ C: second step when the
        // speculative record is the one the sequential algorithm reads next
        const bool hit = go1 && v1 == svox;
        my_spec += hit ? 1u : 0u;
        const bool out2 = hit && sv.outside();
        why = out2 ? kEndMask : why;
        commit_if(hit && !out2, c1x, c1y, c1z, v1);
        const bool live2 = hit && !out2;
        float c2x, c2y, c2z;
        uint32_t v2;
        int i2x, i2y, i2z;
        const bool go2 = step(sv, live2, c2x, c2y, c2z, v2, i2x, i2y, i2z);
        // pending candidate for the next iteration
        alive = hit ? go2 : go1;
        pend = alive;
        const int jx = hit ? i2x : i1x, jy = hit ? i2y : i1y, jz = hit ? i2z : i1z;
        gvox = alive ? (hit ? v2 : v1) : gvox;
        if (BL != 0) grv = alive ? recv(jx, jy, jz, gvox) : grv;
    }

    // ---- counters: one atomic per warp
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        my_steps += __shfl_xor_sync(kFull, my_steps, o);
        my_particles += __shfl_xor_sync(kFull, my_particles, o);
        my_active += __shfl_xor_sync(kFull, my_active, o);
        my_spec += __shfl_xor_sync(kFull, my_spec, o);
    }
    if (lane == 0) {
        atomicAdd(a.stats + kStatSteps, (unsigned long long)my_steps);
        atomicAdd(a.stats + kStatParticles, (unsigned long long)my_particles);
        atomicAdd(a.stats + kStatLaneActive, (unsigned long long)my_active);
        atomicAdd(a.stats + kStatLaneSlots, (unsigned long long)iters * 32ull);
        atomicAdd(a.stats + kStatSpecHits, (unsigned long long)my_spec);
    }
}

template <int F, bool HALF, bool OUT, int BL>
cudaError_t launch_sb(const TrackArgs& a, int num_sms, cudaStream_t st) {
    auto k = track_spec_kernel<F, HALF, OUT, BL>;
    if (a.nparticles == 0) return cudaSuccess;
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kSpecThreads, 0);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    const uint64_t need = (a.nparticles + (uint64_t)kSpecThreads - 1) / (uint64_t)kSpecThreads;
    const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
    const unsigned grid = (unsigned)(need < full ? need : full);
    k<<<grid, kSpecThreads, 0, st>>>(a);
    return cudaGetLastError();
}

template <int F, bool HALF>
cudaError_t launch_sf(const TrackArgs& a, int num_sms, cudaStream_t st) {
    const bool out = a.o_nsteps || a.o_reason || a.o_end || a.o_paths || a.conn;
    if (a.rb_log == 0)
        return out ? launch_sb<F, HALF, true, 0>(a, num_sms, st) : launch_sb<F, HALF, false, 0>(a, num_sms, st);
    if (a.rb_log == kBrickLog)
        return out ? launch_sb<F, HALF, true, kBrickLog>(a, num_sms, st)
                   : launch_sb<F, HALF, false, kBrickLog>(a, num_sms, st);
    return cudaErrorInvalidValue;
}

}  // namespace

cudaError_t launch_track_spec(const TrackArgs& a, int nfibres, bool half, int num_sms, cudaStream_t st) {
    switch (nfibres * 2 + (half ? 1 : 0)) {
        case 2: return launch_sf<1, false>(a, num_sms, st);
        case 3: return launch_sf<1, true>(a, num_sms, st);
        case 4: return launch_sf<2, false>(a, num_sms, st);
        case 5: return launch_sf<2, true>(a, num_sms, st);
        case 6: return launch_sf<3, false>(a, num_sms, st);
        case 7: return launch_sf<3, true>(a, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace pt
