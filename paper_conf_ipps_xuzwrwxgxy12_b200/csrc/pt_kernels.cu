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
// path lengths are exponentially distributed.  A round is 3 x PT_ROUND_BLOCKS
// steps (default 6): each Philox block supplies three sample indices (R16); the first is
// computed at the round start, the next one before the round's 3rd step.  The gather of
// the next step's record doubles as the mask test of the candidate voxel (sentinel records,
// R11); the round's last gather is deferred to the next round's start, where it is issued
// by the same instruction as the first gather of freshly refilled lanes.
#include <cuda_runtime.h>
#include <cub/device/device_radix_sort.cuh>

#include <cstdint>

#include "pt_claim.cuh"
#include "pt_device.cuh"
#include "pt_internal.h"

#ifndef PT_RUNLEN
#define PT_RUNLEN 1  // merge consecutive visits of a voxel before the RED (0: ablation iv, one RED per step;
                     // 2: ablation iv, run-length merge + warp aggregation of same-voxel flushes)
#endif
#ifndef PT_REFILL_MIN
#define PT_REFILL_MIN 2  // free lanes a warp waits for before refilling (amortises the refill block)
#endif
#ifndef PT_CTA_MINB
#define PT_CTA_MINB 1  // resident CTAs per SM the persistent kernel is compiled for (occupancy sweeps)
#endif
#ifndef PT_ROUND_BLOCKS
#define PT_ROUND_BLOCKS 2  // Philox blocks (3 steps each) per refill round: 6-step rounds (1: 0.99x, 3: 1.00x)
#endif
#ifndef PT_REC_AFFINE
#define PT_REC_AFFINE 0  // brick position as a sum of per-axis affine terms (experiment builds: 1)
#endif
#ifndef PT_SLOTS
#define PT_SLOTS 1  // particles per lane in the persistent kernel (1 or 2; 2 measured no faster)
#endif

namespace pt {

enum { kEndMask = 0, kEndCurv = 1, kEndMaxlen = 2 };

// State of one particle slot of a lane.
template <int F, bool HALF>
struct Slot {
    bool alive;        // holds a particle in flight
    bool pend;         // the round's 3rd candidate step waits for the next round's gather
    float qx, qy, qz;  // committed position, centred coordinates (R10)
    float px, py, pz;  // direction of the last (candidate) step
    uint32_t gvox;     // voxel read by the round-start gather (seed or pending candidate)
    uint32_t grv;      // its position in the record volume (rec_vox)
    int n;             // committed steps
    uint64_t pid;      // global particle id = seed_id * P + j (RNG key, R16)
    uint32_t run_vox, run_cnt;  // run-length merge of consecutive visits
    uint32_t sfix;     // paper mode (NEXT-1): the particle's sample volume, j mod S
    int why;           // >= 0: ended with this reason, outputs pending (finish)
    uint4 W;           // Philox block of the current round
    Rec<F, HALF> rv;   // record of the current step
    uint64_t tmask;    // NEXT-2: targets entered by the path so far (bit t-1)
    uint32_t sidx;     // NEXT-2: seed index of this call
};

template <bool REFILL, int SLOTS>
struct Cta {
    static constexpr int kTPB = REFILL ? (SLOTS == 2 ? kThreads2 : kThreads) : kSimpleThreads;
};

// The tracking kernel.  OUT: per-particle outputs or polylines are recorded (compiled out of
// the bench path).  REFILL: persistent CTAs with lane refill (false: one particle per thread,
// the no-refill ablation).  SLOTS: particles per lane; with 2, a lane interleaves the steps
// of two independent particles so that one particle's gather is in flight while the other
// computes (more gathers in flight per SM without more threads, all from the same claim).
// BL: record layout, log2 brick edge (0 = raster), a compile-time constant so
// the record position costs a few shift/mask instructions with immediates.
template <int F, bool HALF, bool REFILL, bool OUT, int SLOTS, int BL>
__global__ void __launch_bounds__(Cta<REFILL, SLOTS>::kTPB, REFILL ? PT_CTA_MINB : 1) track_kernel(const __grid_constant__ TrackArgs a) {
    using R = Rec<F, HALF>;
    constexpr int RB = R::kBytes;
    constexpr int TPB = Cta<REFILL, SLOTS>::kTPB;
    __shared__ unsigned long long s_li[OUT ? SLOTS * TPB : 1];  // particle index (outputs)
    __shared__ uint32_t s_q[TPB / 32][3];                        // per-warp sub-chunk
    __shared__ unsigned long long s_work;                        // CTA claim + tickets
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t wib = threadIdx.x >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const bool has_map = a.map != nullptr;
    // privatised map copies (PT_MAP_COPIES): CTA b adds into copy b % map_copies
    uint32_t* const map = has_map ? a.map + (size_t)(blockIdx.x % a.map_copies) * ((size_t)a.nx * a.ny * a.nz)
                                  : nullptr;
    if (threadIdx.x == 0) s_work = kNoChunk << 24;
    if (lane == 0) {
        s_q[wib][0] = 0u;
        s_q[wib][1] = 0u;
        s_q[wib][2] = 0u;
    }
    __syncthreads();

    Slot<F, HALF> P[SLOTS];
#pragma unroll
    for (int sl = 0; sl < SLOTS; ++sl) {
        P[sl].alive = false;
        P[sl].pend = false;
        P[sl].qx = P[sl].qy = P[sl].qz = 0.f;
        P[sl].px = P[sl].py = P[sl].pz = 0.f;
        P[sl].gvox = 0u;
        P[sl].grv = 0u;
        P[sl].n = 0;
        P[sl].pid = 0ull;
        P[sl].run_vox = 0u;
        P[sl].run_cnt = 0u;
        P[sl].sfix = 0u;
        P[sl].why = -1;
        P[sl].W = make_uint4(0u, 0u, 0u, 0u);
        P[sl].tmask = 0ull;
        P[sl].sidx = 0u;
#pragma unroll
        for (int k = 0; k < R::kWords; ++k) P[sl].rv.w[k] = 0u;
    }
    // per-lane counters (a lane never sees 2^32 steps in one launch)
    uint32_t my_steps = 0, my_particles = 0, my_active = 0, rounds = 0;
    bool exhausted = false;  // warp-uniform

    // position of voxel (ix, iy, iz) = raster index v in the record volume (rec_vox)
#if PT_REC_AFFINE
    // rec_vox as a sum of per-axis terms: with b = BL and u = u_b * 2^b + (u & m),
    //   (x & m) = x - 2^b x_b, (y & m) << b = 2^b y - 2^2b y_b, (z & m) << 2b = 2^2b z - 2^3b z_b,
    // so rec_vox = x + x_b Kx + 2^b y + y_b Ky + 2^2b z + z_b Kz (mod 2^32; the exact value
    // is < 2^32, checked at load) with the constants below
    const uint32_t rKx = (1u << (3 * BL)) - (1u << BL);
    const uint32_t rKy = (a.rb_nbx << (3 * BL)) - (1u << (2 * BL));
    const uint32_t rKz = ((a.rb_nbx * a.rb_nby) << (3 * BL)) - (1u << (3 * BL));
#endif
    auto recv = [&](int ix, int iy, int iz, uint32_t v) -> uint32_t {
        if (BL == 0) return v;
#if PT_REC_AFFINE
        {
            const uint32_t x = (uint32_t)ix, y = (uint32_t)iy, z = (uint32_t)iz;
            uint32_t r = x + (x >> BL) * rKx;
            r += (y >> BL) * rKy + (y << BL);
            r += (z >> BL) * rKz + (z << (2 * BL));
            return r;
        }
#endif
        constexpr uint32_t m = (1u << BL) - 1u;
        const uint32_t x = (uint32_t)ix, y = (uint32_t)iy, z = (uint32_t)iz;
        const uint32_t br = ((z >> BL) * a.rb_nby + (y >> BL)) * a.rb_nbx + (x >> BL);
        return (br << (3 * BL)) | ((z & m) << (2 * BL)) | ((y & m) << BL) | (x & m);
    };
    // a termination only records the reason; outputs and the count flush are written once
    // per round for all ended particles at the top of the loop
    auto end = [&](Slot<F, HALF>& x, int w) {
        x.why = w;
        x.alive = false;
        x.pend = false;
    };
    // SetEndPoint()
    auto finish = [&](Slot<F, HALF>& x, int sl) {
        if (OUT && (a.o_nsteps || a.o_reason || a.o_end)) {
            const uint64_t li = s_li[sl * TPB + threadIdx.x];
            if (a.o_nsteps) a.o_nsteps[li] = (uint16_t)x.n;
            if (a.o_reason) a.o_reason[li] = (uint8_t)x.why;
            if (a.o_end) {
                float* e = a.o_end + 3 * li;
                e[0] = __fadd_rn(x.qx, a.fcx);
                e[1] = __fadd_rn(x.qy, a.fcy);
                e[2] = __fadd_rn(x.qz, a.fcz);
            }
        }
        if (has_map && x.run_cnt) atomicAdd(map + x.run_vox, x.run_cnt);  // RED
        x.run_cnt = 0;
        if (OUT && a.conn) {  // NEXT-2: one count per target the streamline entered
            uint64_t m = x.tmask;
            while (m) {
                const int t = __ffsll((long long)m) - 1;
                atomicAdd(a.conn + (uint64_t)x.sidx * a.ntargets + (uint32_t)t, 1u);
                m &= m - 1ull;
            }
            x.tmask = 0ull;
        }
        my_steps += (uint32_t)x.n;
        my_particles += 1u;
        x.why = -1;
    };
    // commit a step (if c): new position, one visit of the new voxel (R13);
    // consecutive visits of the same voxel are merged (run length) and flushed with a
    // predicated RED when the voxel changes.  Straight-line, no branch.
    auto commit_if = [&](Slot<F, HALF>& x, int sl, bool c, float nx_, float ny_, float nz_, uint32_t v) {
        x.qx = c ? nx_ : x.qx;
        x.qy = c ? ny_ : x.qy;
        x.qz = c ? nz_ : x.qz;
        x.n += c ? 1 : 0;
        if (has_map) {
#if PT_RUNLEN == 2
            // lanes flushing the same voxel form one group (__match_any_sync); the group's
            // lowest lane issues one RED with the group's summed count (labelled-partition
            // reduction: every lane of a group passes the same member mask)
            const bool change = v != x.run_vox;
            const bool fl = c && change && x.run_cnt != 0u;
            const uint32_t grp = __match_any_sync(kFull, fl ? x.run_vox : 0xFFFFFFFFu);
            const uint32_t sum = __reduce_add_sync(grp, fl ? x.run_cnt : 0u);
            red_add_if(fl && lane == (uint32_t)(__ffs(grp) - 1), map + x.run_vox, sum);
            x.run_cnt = c ? (change ? 1u : x.run_cnt + 1u) : x.run_cnt;
            x.run_vox = c ? v : x.run_vox;
#elif PT_RUNLEN
            const bool change = v != x.run_vox;
            red_add_if(c && change && x.run_cnt != 0u, map + x.run_vox, x.run_cnt);
            x.run_cnt = c ? (change ? 1u : x.run_cnt + 1u) : x.run_cnt;
            x.run_vox = c ? v : x.run_vox;
#else
            red_add_if(c, map + v, 1u);  // ablation (iv): one global RED per committed step
#endif
        }
        if (OUT && a.conn && c) {  // NEXT-2: targets entered by committed steps (R21)
            const uint32_t lbl = __ldg(a.labels + v);
            x.tmask |= lbl ? (1ull << (lbl - 1u)) : 0ull;
        }
        if (OUT && a.o_paths && c && x.n < a.path_stride) {
            float* pp = a.o_paths + (s_li[sl * TPB + threadIdx.x] * (uint64_t)a.path_stride + (uint64_t)x.n) * 3u;
            pp[0] = __fadd_rn(x.qx, a.fcx);
            pp[1] = __fadd_rn(x.qy, a.fcy);
            pp[2] = __fadd_rn(x.qz, a.fcz);
        }
    };
    // GetStartPoint(): centred seed position, seed voxel (R10, R12)
    auto start = [&](Slot<F, HALF>& x, int sl, uint64_t si, uint64_t j) {
        const uint64_t li = si * a.P + j;
        if (OUT) s_li[sl * TPB + threadIdx.x] = li;
        const uint64_t sid = a.seed_ids ? a.seed_ids[si] : si;
        x.pid = sid * a.P + j;
        x.sfix = a.sample_mode ? (uint32_t)(j % a.S) : 0u;
        x.tmask = 0ull;
        x.sidx = (uint32_t)si;
        x.qx = __fsub_rn(a.seeds[3 * si + 0], a.fcx);
        x.qy = __fsub_rn(a.seeds[3 * si + 1], a.fcy);
        x.qz = __fsub_rn(a.seeds[3 * si + 2], a.fcz);
        x.n = 0;
        x.pend = false;
        x.run_cnt = 0;
        x.alive = true;
        if (OUT && a.o_paths) {
            float* pp = a.o_paths + li * (uint64_t)a.path_stride * 3u;
            pp[0] = __fadd_rn(x.qx, a.fcx);
            pp[1] = __fadd_rn(x.qy, a.fcy);
            pp[2] = __fadd_rn(x.qz, a.fcz);
        }
        const int ix = axis_index(x.qx, a.cx), iy = axis_index(x.qy, a.cy), iz = axis_index(x.qz, a.cz);
        if ((unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz) {
            x.gvox = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
            x.grv = recv(ix, iy, iz, x.gvox);
        } else {
            end(x, kEndMask);  // seed outside the volume (R12): finished right away, so the
            finish(x, sl);     // refill loop may hand this lane another particle
        }
    };
    // one step of Alg. 1's inner loop for a slot; k = position in the round
    auto step = [&](Slot<F, HALF>& x, int sl, int k) {
        my_active += x.alive ? 1u : 0u;
        const bool first = x.n == 0;
        // choose the fibre closest to the previous direction: eligible iff
        // f_j > fib_thr (R7), strict >, lowest j wins (R8); the first step takes fibre 0
        // (R5).  "Interpolation()" of Alg. 1 = this sample's record at the voxel (R2).
        float vx, vy, vz, f0;
        x.rv.fibre(0, vx, vy, vz, f0);
        float bc = __fadd_rn(__fadd_rn(__fmul_rn(vx, x.px), __fmul_rn(vy, x.py)), __fmul_rn(vz, x.pz));
        float best = f0 > a.fib_thr ? fabsf(bc) : -1.f;
#pragma unroll
        for (int j = 1; j < F; ++j) {
            float ux, uy, uz, fu;
            x.rv.fibre(j, ux, uy, uz, fu);
            const float cj = __fadd_rn(__fadd_rn(__fmul_rn(ux, x.px), __fmul_rn(uy, x.py)), __fmul_rn(uz, x.pz));
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
        const bool neg = first ? (x.W.w >> 31) != 0u : !(bc > 0.f);
        // StepToNextPoint(): q' = q + h * (sign * v), no FMA
        const float dx = neg ? -vx : vx, dy = neg ? -vy : vy, dz = neg ? -vz : vz;
        const float nqx = __fadd_rn(x.qx, __fmul_rn(a.step, dx));
        const float nqy = __fadd_rn(x.qy, __fmul_rn(a.step, dy));
        const float nqz = __fadd_rn(x.qz, __fmul_rn(a.step, dz));
        const int ix = axis_index(nqx, a.cx), iy = axis_index(nqy, a.cy), iz = axis_index(nqz, a.cz);
        const bool inb = (unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz;
        const uint32_t v = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
        // stop criteria in order: maximum steps (R14), angle, volume (R11)
        const bool maxed = x.n == a.max_steps;
        const bool go = x.alive && !maxed && curv_ok && inb;
        x.why = (x.alive && !go) ? (maxed ? kEndMaxlen : (!curv_ok ? kEndCurv : kEndMask)) : x.why;
        x.alive = go;
        x.px = go ? dx : x.px;
        x.py = go ? dy : x.py;
        x.pz = go ? dz : x.pz;
        if (k < 3 * PT_ROUND_BLOCKS - 1) {
            if ((k + 1) % 3 == 0) {
                // the next step opens the round's next Philox block: a live lane has
                // committed t0 + k steps, so that block is (n + 1) / 3 (R16)
                x.W = philox4x32_10(make_uint4(((uint32_t)x.n + 1u) / 3u, (uint32_t)x.pid, (uint32_t)(x.pid >> 32), 0u),
                                    a.key0, a.key1);
            }
            const uint32_t w = ((k + 1) % 3 == 0) ? x.W.x : ((k + 1) % 3 == 1) ? x.W.y : x.W.z;
            const uint32_t sk = a.sample_mode ? x.sfix : sample_of(w, a.S);
            const uint32_t rvx = recv(ix, iy, iz, v);
            ldg_record_if<RB>(go, a.rec + ((uint64_t)rvx * a.S + sk) * RB, x.rv.w);
            const bool outside = go && x.rv.outside();  // candidate outside the mask (R11)
            x.why = outside ? kEndMask : x.why;
            x.alive = go && !outside;
            commit_if(x, sl, x.alive, nqx, nqy, nqz, v);
        } else {
            x.pend = go;  // next round's start gathers and tests it
            x.gvox = go ? v : x.gvox;
            if (BL != 0) x.grv = go ? recv(ix, iy, iz, v) : x.grv;
        }
    };

    if (!REFILL) {
        const uint64_t g = (uint64_t)blockIdx.x * TPB + threadIdx.x;
        if (g < a.nparticles) {
            const uint64_t si = g / a.P;
            start(P[0], 0, si, g - si * a.P);
        }
    }

    for (;;) {
#pragma unroll
        for (int sl = 0; sl < SLOTS; ++sl)
            if (P[sl].why >= 0) finish(P[sl], sl);  // particles that ended in the last round

        // ------------------------------------------------ lane refill (replaces the
        // paper's CPU Reduction()/segment relaunch)
        if (REFILL) {
            // refill once at least PT_REFILL_MIN slots of the warp are free (or none is live)
            uint32_t nfree = 0;
#pragma unroll
            for (int sl = 0; sl < SLOTS; ++sl) nfree += (uint32_t)__popc(__ballot_sync(kFull, !P[sl].alive));
            if (!exhausted && nfree != 0u && (nfree >= (uint32_t)PT_REFILL_MIN || nfree == 32u * SLOTS)) {
                uint32_t cseed = s_q[wib][0], cnext = s_q[wib][1], cend = s_q[wib][2];
#pragma unroll
                for (int sl = 0; sl < SLOTS; ++sl) {
                    uint32_t need = __ballot_sync(kFull, !P[sl].alive);
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
                        if (!P[sl].alive && rank < avail) start(P[sl], sl, cseed, (uint64_t)(cnext + rank));
                        const uint32_t cnt = (uint32_t)__popc(need);
                        cnext += cnt < avail ? cnt : avail;
                        need = __ballot_sync(kFull, !P[sl].alive);
                    }
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
        bool any_alive = false;
#pragma unroll
        for (int sl = 0; sl < SLOTS; ++sl) any_alive |= P[sl].alive;
        if (!__any_sync(kFull, any_alive)) break;
        rounds += 1u;

        // ------------------------------------------------ round start: one Philox block per
        // slot, gather of (pending candidate | seed) voxel = mask test + first step's record;
        // the slots' gathers are issued back to back so they are in flight together
#pragma unroll
        for (int sl = 0; sl < SLOTS; ++sl) {
            Slot<F, HALF>& x = P[sl];
            const uint32_t t0 = (uint32_t)x.n + (x.pend ? 1u : 0u);  // a multiple of 3
            x.W = philox4x32_10(make_uint4(t0 / 3u, (uint32_t)x.pid, (uint32_t)(x.pid >> 32), 0u), a.key0, a.key1);
            const uint32_t s0 = a.sample_mode ? x.sfix : sample_of(x.W.x, a.S);
            ldg_record_if<RB>(x.alive, a.rec + ((uint64_t)(BL == 0 ? x.gvox : x.grv) * a.S + s0) * RB, x.rv.w);
        }
#pragma unroll
        for (int sl = 0; sl < SLOTS; ++sl) {
            Slot<F, HALF>& x = P[sl];
            // seed outside the mask (R12) or pending candidate rejected (R11)
            const bool outside = x.alive && x.rv.outside();
            x.why = outside ? kEndMask : x.why;
            x.alive = x.alive && !outside;
            // accepted candidate: recomputed bit-identically from (q, d) instead of kept
            commit_if(x, sl, x.pend && !outside, __fadd_rn(x.qx, __fmul_rn(a.step, x.px)),
                      __fadd_rn(x.qy, __fmul_rn(a.step, x.py)), __fadd_rn(x.qz, __fmul_rn(a.step, x.pz)), x.gvox);
            x.pend = false;
        }

        // ------------------------------------------------ 3 x PT_ROUND_BLOCKS steps, slots interleaved
#pragma unroll
        for (int k = 0; k < 3 * PT_ROUND_BLOCKS; ++k) {
#pragma unroll
            for (int sl = 0; sl < SLOTS; ++sl) step(P[sl], sl, k);
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
        atomicAdd(a.stats + kStatLaneSlots, (unsigned long long)rounds * (3ull * PT_ROUND_BLOCKS) * 32ull * SLOTS);
    }
}

// ------------------------------------------------------------------------- repack
// Canonical [F][S][Z][Y][X](x3) sample volumes -> rec[vox][s] (one thread per record,
// s fastest so the record stores are coalesced).  Voxels outside the mask get the
// sentinel f0 = all-ones; non-finite values inside the mask are counted in *bad.
template <bool HALF>
__global__ void repack_kernel(const void* __restrict__ dyads, const void* __restrict__ fr,
                              const uint8_t* __restrict__ mask, uint8_t* __restrict__ rec,
                              int nx, int ny, int64_t V, RecLayout L, int S, int F, int RB,
                              unsigned long long* bad) {
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
        const uint64_t rv = rec_vox_raster((uint32_t)vox, (uint32_t)nx, (uint32_t)ny, L.b, L.nbx, L.nby);
        uint8_t* out = rec + (rv * (uint64_t)S + (uint64_t)s) * RB;
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
template <int F, bool HALF, bool REFILL, bool OUT, int BL>
static cudaError_t launch_tb(const TrackArgs& a, int num_sms, cudaStream_t st) {
    constexpr int SL = REFILL ? PT_SLOTS : 1;
    auto k = track_kernel<F, HALF, REFILL, OUT, SL, BL>;
    constexpr int TPB = Cta<REFILL, SL>::kTPB;
    if (a.nparticles == 0) return cudaSuccess;
    unsigned grid;
    if (REFILL) {
        int per_sm = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, TPB, 0);
        if (e != cudaSuccess) return e;
        if (per_sm < 1) return cudaErrorInvalidConfiguration;
        const uint64_t need = (a.nparticles + (uint64_t)TPB * SL - 1) / ((uint64_t)TPB * SL);
        const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
        grid = (unsigned)(need < full ? need : full);
    } else {
        grid = (unsigned)((a.nparticles + TPB - 1) / TPB);
    }
    k<<<grid, TPB, 0, st>>>(a);
    return cudaGetLastError();
}

// record layouts compiled into the tracking kernel: raster and 16^3 bricks
template <int F, bool HALF, bool REFILL, bool OUT>
static cudaError_t launch_t(const TrackArgs& a, int num_sms, cudaStream_t st) {
    if (a.rb_log == 0) return launch_tb<F, HALF, REFILL, OUT, 0>(a, num_sms, st);
    if (a.rb_log == kBrickLog) return launch_tb<F, HALF, REFILL, OUT, kBrickLog>(a, num_sms, st);
    return cudaErrorInvalidValue;
}

template <int F, bool HALF>
static cudaError_t launch_f(const TrackArgs& a, bool simple, int num_sms, cudaStream_t st) {
    const bool out = a.o_nsteps || a.o_reason || a.o_end || a.o_paths || a.conn;
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

RecLayout rec_layout(int nx, int ny, int nz, uint32_t b) {
    RecLayout L;
    const uint32_t e = 1u << b;
    L.b = b;
    L.nbx = ((uint32_t)nx + e - 1u) >> b;
    L.nby = ((uint32_t)ny + e - 1u) >> b;
    L.nbz = ((uint32_t)nz + e - 1u) >> b;
    return L;
}

cudaError_t launch_repack(const void* dyads, const void* f, const uint8_t* mask, uint8_t* rec,
                          int nx, int ny, int nz, const RecLayout& L, int S, int F, bool half, int rec_bytes,
                          unsigned long long* bad, cudaStream_t st) {
    const int64_t V = (int64_t)nx * ny * nz;
    const int64_t total = V * (int64_t)S;
    int64_t blocks = (total + 255) / 256;
    if (blocks > 148 * 64) blocks = 148 * 64;
    if (blocks < 1) blocks = 1;
    if (half)
        repack_kernel<true><<<(unsigned)blocks, 256, 0, st>>>(dyads, f, mask, rec, nx, ny, V, L, S, F, rec_bytes, bad);
    else
        repack_kernel<false><<<(unsigned)blocks, 256, 0, st>>>(dyads, f, mask, rec, nx, ny, V, L, S, F, rec_bytes, bad);
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
