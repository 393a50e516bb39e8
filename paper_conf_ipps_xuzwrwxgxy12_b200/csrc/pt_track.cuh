// pt_track.cuh -- the particle-stepping kernel of the probabilistic-streamlining hot path
// (sm_100a): Algorithm 1's inner loop with the semantics of P:L98-121 and the
// readings of DESIGN.md (contract C-ALG, R1-R24).  One template, instantiated per fibre
// count / record precision in pt_track_f{1,2,3}.cu so the three files compile in parallel.
//
//   REFILL  persistent CTAs, one per SM, warps pull 32-particle sub-chunks from a global
//           work queue (pt_claim.cuh) and refill dead lanes with a ballot/popc prefix at
//           the start of every round, so the warp stays converged while path lengths are
//           exponentially distributed.  false: one particle per thread and
//           no refill -- the paper's "Extreme case 1", ablation (i).
//   OUT     per-particle outputs / polylines / the seed x target matrix are recorded
//           (compiled out of the bench path).
//   BL      record layout, log2 brick edge (0 raster, 4 = 16^3 bricks) as a compile-time
//           constant, or -1: read from the launch arguments.  The compile-time layouts are
//           the bench path and assume the random-sample mode (R1); paper mode (NEXT-1,
//           sample_mode = 1) runs the BL = -1 instantiations.
//   VM      NEXT-3 FSL-fidelity variants compiled in (bit mask; 0 = the north star's
//           semantics): kVarBidir R22 bidirectional streamlines (half 1 restarts in the same
//           lane at a round boundary), kVarInterp R23 probabilistic interpolation of the
//           sampled voxel (one extra Philox block per step, stream 2 + half, plus a 1-byte
//           mask read of the candidate's nearest voxel), kVarInit R24 random / f-weighted
//           first fibre.  Each compiled-in variant is still switched by its launch argument
//           (bidir / interp / init_mode), so VM = kVarAll runs any combination.
//   UNQ     NEXT-2 per-streamline-unique visitation map (R25): a voxel counts once
//           per streamline; exact, through a per-lane open-addressing hash set of the
//           voxels the streamline has entered (global scratch, generation-tagged).
//
// A round is 3 x kRoundBlocks steps (6): each Philox block supplies three sample indices
// (R16); the first is computed at the round start, the next one before the round's 3rd
// step.  The gather of the next step's record doubles as the mask test of the candidate
// voxel (sentinel records, R11); the round's last gather is deferred to the next round's
// start, where it is issued by the same instruction as the first gather of refilled lanes.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "pt_claim.cuh"
#include "pt_device.cuh"
#include "pt_internal.h"

#ifndef PT_REC_AFFINE
#define PT_REC_AFFINE 1  // brick position of the bench layout as per-axis terms (0: the bit-field form)
#endif
#ifndef PT_RUNLEN
#define PT_RUNLEN 1  // merge consecutive visits of a voxel before the RED (0: ablation iv, one RED per step)
#endif
#ifndef PT_REFILL_MIN
#define PT_REFILL_MIN 2  // free lanes a warp waits for before refilling (amortises the refill block)
#endif

namespace pt {

enum { kEndMask = 0, kEndCurv = 1, kEndMaxlen = 2 };
constexpr int kRoundBlocks = 2;             // Philox blocks per refill round (6-step rounds)
constexpr int kRoundSteps = 3 * kRoundBlocks;

// R23: per axis, the upper of the two voxels whose centres bracket q is taken with
// probability = its linear weight (t = q - 0.5, m = floor(t), fr = t - m, r = (w>>8) 2^-24).
__device__ __forceinline__ int interp_axis(float q, int c, uint32_t w) {
    const float t = __fsub_rn(q, 0.5f);
    const float m = floorf(t);
    const float fr = __fsub_rn(t, m);
    const float r = __fmul_rn(__uint2float_rn(w >> 8), 0x1p-24f);
    return c + __float2int_rz(m) + (r < fr ? 1 : 0);
}

// State of the particle a lane owns.
enum { kVarBidir = 1, kVarInterp = 2, kVarInit = 4, kVarAll = 7 };

template <int F, bool HALF, bool UNQ>
struct Lane {
    bool alive;        // holds a particle (half) in flight
    bool pend;         // the round's last candidate step waits for the next round's gather
    float qx, qy, qz;  // committed position, centred coordinates (R10)
    float px, py, pz;  // direction of the last (candidate) step (fp32 records)
    uint32_t pxy, pzw; // the same as packed halves (fp16 records, see hdot)
    uint32_t gvox;     // raster voxel of the round-start gather (seed or pending candidate)
    uint32_t grv;      // its position in the record volume (rec_vox)
    int n;             // committed steps (of this half)
    uint64_t pid;      // global particle id = seed_id * P + j (RNG key, R16)
    uint32_t run_vox, run_cnt;  // run-length merge of consecutive visits (UNQ: current voxel)
    uint32_t sfix;     // paper mode (NEXT-1): the particle's sample volume, j mod S
    int why;           // >= 0: ended with this reason, outputs pending (finish)
    uint4 W;           // Philox block of the current round (stream = half)
    Rec<F, HALF> rv;   // record of the current step
    uint64_t tmask;    // NEXT-2: targets entered by the streamline so far (bit t-1)
    uint32_t sidx;     // seed index of this call
    // variants (R22, R24)
    uint32_t half;     // 0, or 1 = the reverse half of a bidirectional streamline
    bool have_d0;      // half 0 computed its first direction
    float d0x, d0y, d0z;
    uint32_t d0xy, d0zw;  // (fp16 records)
    uint32_t winit;    // word 3 of Philox(stream 2, block 0): the first fibre (R24)
    // UNQ (R25)
    uint32_t gen;      // generation tag of the streamline in the lane's hash set
    uint32_t prev_vox; // the voxel entered before run_vox (recent-voxel filter)
    bool upend;        // a probe of the hash set is in flight for voxel ukey ...
    uint32_t ukey, uh; // ... at slot uh,
    unsigned long long ue;  // whose entry the in-flight load returns
};

// CTA size: one CTA per SM; the variant / unique instantiations keep more state per lane
// and run 768 threads (<= 85 registers) instead of 1024 (<= 64)
template <bool REFILL, int VM, bool UNQ>
__host__ __device__ constexpr int track_tpb() {
    return REFILL ? (((VM & (kVarInterp | kVarInit)) != 0 || UNQ) ? kThreadsExt : kThreads) : kSimpleThreads;
}

template <int F, bool HALF, bool REFILL, bool OUT, int BL, int VM, bool UNQ, bool NB = false>
__global__ void __launch_bounds__(track_tpb<REFILL, VM, UNQ>(), 1) track_kernel(const __grid_constant__ TrackArgs a) {
    using R = Rec<F, HALF>;
    using L = Lane<F, HALF, UNQ>;
    constexpr int RB = R::kBytes;
    constexpr int TPB = track_tpb<REFILL, VM, UNQ>();
    constexpr bool VB = (VM & kVarBidir) != 0, VI = (VM & kVarInterp) != 0, VN = (VM & kVarInit) != 0;
    // q and d of a particle that ends are read again only for its outputs (end point, path)
    constexpr bool KEEPQ = OUT;
    // the bench instantiations key the map by the record voxel (track_rv_keys): no raster
    // voxel index on their path
    constexpr bool RVKEY = PT_RVKEYS && BL > 0 && !OUT && !UNQ && VM == 0 && REFILL;
    // ... and with margin bricks (PT_REC_MARGIN; launched only when a.nobounds) skip the
    // bounds test of every candidate
    constexpr bool NOB = PT_REC_MARGIN && RVKEY && NB;
    __shared__ unsigned long long s_li[OUT ? TPB : 1];  // particle index (outputs)
    __shared__ uint32_t s_q[TPB / 32][3];               // per-warp sub-chunk
    __shared__ unsigned long long s_work;               // CTA claim + tickets
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t wib = threadIdx.x >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    // the map is raster-ordered (a record-ordered map was measured 6 % slower)
    uint32_t* const map = a.map;
    const bool has_map = map != nullptr;
    const uint32_t H = (VB && a.bidir) ? 2u : 1u;      // output entries per particle
    const bool interp = VI && a.interp;
    const uint32_t init_mode = VN ? a.init_mode : 0u;
    const bool smode = BL < 0 && a.sample_mode != 0u;  // paper mode (NEXT-1): s = j mod S
    if (threadIdx.x == 0) s_work = kNoChunk << 24;
    if (lane == 0) {
        s_q[wib][0] = 0u;
        s_q[wib][1] = 0u;
        s_q[wib][2] = 0u;
    }
    __syncthreads();
    // UNQ: this lane's hash set (2^ulog generation-tagged entries, zeroed by pt_track)
    unsigned long long* const utab =
        UNQ ? a.utab + (((uint64_t)blockIdx.x * TPB + threadIdx.x) << a.ulog) : nullptr;
    if (UNQ) PT_BOUND(a, (uint64_t)blockIdx.x * TPB + threadIdx.x < a.utab_lanes);

    L x;
    x.alive = false;
    x.pend = false;
    x.qx = x.qy = x.qz = 0.f;
    x.px = x.py = x.pz = 0.f;
    x.pxy = x.pzw = 0u;
    x.d0xy = x.d0zw = 0u;
    x.gvox = 0u;
    x.grv = 0u;
    x.n = 0;
    x.pid = 0ull;
    x.run_vox = 0u;
    x.run_cnt = 0u;
    x.sfix = 0u;
    x.why = -1;
    x.W = make_uint4(0u, 0u, 0u, 0u);
    x.tmask = 0ull;
    x.sidx = 0u;
    x.half = 0u;
    x.have_d0 = false;
    x.d0x = x.d0y = x.d0z = 0.f;
    x.winit = 0u;
    x.gen = 0u;
    x.prev_vox = 0xFFFFFFFFu;
    x.upend = false;
    x.ukey = x.uh = 0u;
    x.ue = 0ull;
#pragma unroll
    for (int k = 0; k < R::kWords; ++k) x.rv.w[k] = 0u;

    // per-lane counters; flushed to the global counters before they could wrap
    uint32_t my_steps = 0, my_particles = 0, my_active = 0, my_unique = 0, rounds = 0;
    bool exhausted = false;  // warp-uniform

    // position of voxel (ix, iy, iz) = raster index v in the record volume (rec_vox)
    // (recv_p: the same from coordinates already offset by the layout's margin, BL > 0)
    auto recv_p = [&](uint32_t ux, uint32_t uy, uint32_t uz) -> uint32_t {
        constexpr uint32_t b = BL > 0 ? (uint32_t)BL : 1u;
#if PT_REC_AFFINE
        // the same position as a sum of per-axis terms: u_a << (a b) plus (u_a >> b) times
        // the brick stride minus the part of it the shift already counted (a.rb_k*)
        return (ux + (ux >> b) * ((1u << (3 * b)) - (1u << b))) + ((uy << b) + (uy >> b) * a.rb_ky) +
               ((uz << (2 * b)) + (uz >> b) * a.rb_kz);
#else
        constexpr uint32_t m = (1u << b) - 1u;
        const uint32_t br = ((uz >> b) * a.rb_nby + (uy >> b)) * a.rb_nbx + (ux >> b);
        return (br << (3 * b)) | ((uz & m) << (2 * b)) | ((uy & m) << b) | (ux & m);
#endif
    };
    auto recv = [&](int ix, int iy, int iz, uint32_t v) -> uint32_t {
        if (BL == 0) return v;
        if (BL < 0) return rec_vox(ix, iy, iz, a.rb_log, a.rb_nbx, a.rb_nby, a.rb_off);
        const uint32_t o = PT_REC_MARGIN ? a.rb_off : 0u;
        return recv_p((uint32_t)ix + o, (uint32_t)iy + o, (uint32_t)iz + o);
    };
    auto rec_at = [&](uint32_t rv, uint32_t s) -> const uint8_t* {
        return a.rec + rec_slot(rv, s, a.S, BL < 0 ? a.rb_log : (uint32_t)BL) * RB;
    };
    // Philox block of the lane's stream (R16: ctr = {block, pid_lo, pid_hi, stream})
    auto philox = [&](uint32_t block, uint32_t stream) -> uint4 {
        return philox4x32_10(make_uint4(block, (uint32_t)x.pid, (uint32_t)(x.pid >> 32), stream), a.key0, a.key1);
    };
    auto out_index = [&]() -> uint64_t { return OUT ? s_li[threadIdx.x] * H + (VB ? x.half : 0u) : 0ull; };
    // SetEndPoint() of a finished (half-)streamline: outputs, count flush
    auto write_outputs = [&](int n, int why, float qx, float qy, float qz) {
        if (OUT && (a.o_nsteps || a.o_reason || a.o_end)) {
            const uint64_t e = out_index();
            PT_BOUND(a, e < a.out_n);
            if (a.o_nsteps) a.o_nsteps[e] = (uint16_t)n;
            if (a.o_reason) a.o_reason[e] = (uint8_t)why;
            if (a.o_end) {
                float* o = a.o_end + 3 * e;
                o[0] = __fadd_rn(qx, a.fcx);
                o[1] = __fadd_rn(qy, a.fcy);
                o[2] = __fadd_rn(qz, a.fcz);
            }
        }
        my_steps += (uint32_t)n;
    };
    // the whole streamline is done: the connectivity matrix (union of the halves)
    auto particle_done = [&]() {
        if (OUT && a.conn) {  // NEXT-2: one count per target the streamline entered
            uint64_t m = x.tmask;
            while (m) {
                const int t = __ffsll((long long)m) - 1;
                PT_BOUND(a, x.sidx < a.nseeds && (uint32_t)t < a.ntargets);
                atomicAdd(a.conn + (uint64_t)x.sidx * a.ntargets + (uint32_t)t, 1u);
                m &= m - 1ull;
            }
        }
        x.tmask = 0ull;
        my_particles += 1u;
        if (my_steps & 0x80000000u) {  // keep the per-lane sums far from wrapping
            atomicAdd(a.stats + kStatSteps, (unsigned long long)my_steps);
            my_steps = 0u;
        }
    };
    // a run of visits of one voxel: one predicated RED
    auto red_run = [&](bool p, uint32_t vox, uint32_t cnt) {
        if (p) PT_BOUND(a, vox < a.map_keys);
        // (the NOB instantiation is launched only with a permuted scratch map: no select)
        red_add_if(p, map + (NOB ? map_perm(vox, a.map_mask) : map_cell(a, vox)), cnt);
    };
    auto flush_run = [&]() {
        if (!UNQ && has_map) red_run(x.run_cnt != 0u, x.run_vox, x.run_cnt);
        x.run_cnt = 0u;
    };
    // UNQ (R25): has the streamline entered voxel v before?  The lane's hash set answers;
    // the first probe of a voxel entry is only ISSUED when the voxel is entered (its load
    // is in flight while the next step computes and gathers) and RESOLVED at the lane's
    // next voxel entry, or when the half ends -- always before the next probe is issued,
    // so the set seen by every probe is exact.  Collisions continue synchronously.
    auto unq_resolve = [&]() {
        bool fresh = false;
        bool open = x.upend;
        unsigned long long e = x.ue;
        uint32_t h = x.uh;
        const uint32_t mask = (1u << a.ulog) - 1u;
        while (open) {
            PT_BOUND(a, h < (1u << a.ulog));
            if ((uint32_t)(e >> 32) != x.gen) {  // empty or a stale streamline's entry
                utab[h] = ((unsigned long long)x.gen << 32) | x.ukey;
                fresh = true;
                open = false;
            } else if ((uint32_t)e == x.ukey) {
                open = false;
            } else {
                h = (h + 1u) & mask;
                e = utab[h];
            }
        }
        x.upend = false;
        if (has_map && fresh) PT_BOUND(a, x.ukey < a.V);
        red_add_if(has_map && fresh, map + map_cell(a, x.ukey), 1u);
        my_unique += fresh ? 1u : 0u;
    };
    auto unq_issue = [&](bool c, uint32_t v) {
        // the current and the previous voxel are known to be in the set (recent-voxel filter)
        const bool probe = c && v != x.run_vox && v != x.prev_vox;
        if (probe) {
            unq_resolve();
            x.ukey = v;
            x.uh = (v * 0x9E3779B1u) >> (32u - a.ulog);
            x.ue = utab[x.uh];
            x.upend = true;
        }
    };
    // begin half h of the current particle at its seed: centred position, seed voxel.
    // Returns false if the seed is outside the volume (R12).
    auto begin = [&](uint32_t h) -> bool {
        x.half = h;
        PT_BOUND(a, x.sidx < a.nseeds);
        x.qx = __fsub_rn(a.seeds[3 * x.sidx + 0], a.fcx);
        x.qy = __fsub_rn(a.seeds[3 * x.sidx + 1], a.fcy);
        x.qz = __fsub_rn(a.seeds[3 * x.sidx + 2], a.fcz);
        x.n = 0;
        x.pend = false;
        x.run_cnt = 0u;
        x.run_vox = 0xFFFFFFFFu;
        x.prev_vox = 0xFFFFFFFFu;
        if (OUT && a.o_paths) {
            PT_BOUND(a, out_index() < a.out_n && a.path_stride > 0);
            float* pp = a.o_paths + out_index() * (uint64_t)a.path_stride * 3u;
            pp[0] = __fadd_rn(x.qx, a.fcx);
            pp[1] = __fadd_rn(x.qy, a.fcy);
            pp[2] = __fadd_rn(x.qz, a.fcz);
        }
        const int ix = axis_index(x.qx, a.cx), iy = axis_index(x.qy, a.cy), iz = axis_index(x.qz, a.cz);
        // non-finite seeds are outside (a NaN would truncate into the volume)
        const bool fin = isfinite(x.qx) && isfinite(x.qy) && isfinite(x.qz);
        if (fin && (unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz) {
            x.gvox = ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
            x.grv = recv(ix, iy, iz, x.gvox);
            return true;
        }
        return false;
    };
    // a half that ended: outputs; a bidirectional half 0 restarts as half 1 in this lane (R22)
    auto finish = [&]() {
        flush_run();
        if (UNQ) unq_resolve();  // the half's last voxel entry
        write_outputs(x.n, x.why, x.qx, x.qy, x.qz);
        x.why = -1;
        if (VB && H == 2u && x.half == 0u) {
            const bool ok = begin(1u) && x.have_d0;
            if (ok) {  // the reverse half starts against half 0's first direction
                x.px = -x.d0x;
                x.py = -x.d0y;
                x.pz = -x.d0z;
                x.pxy = x.d0xy ^ 0x80008000u;
                x.pzw = x.d0zw ^ 0x00008000u;
                x.alive = true;
                return;
            }
            write_outputs(0, kEndMask, x.qx, x.qy, x.qz);  // seed outside: half 1 is empty too
        }
        particle_done();
    };
    // GetStartPoint(): a new particle (seed index si, particle j of the seed)
    auto start = [&](uint64_t si, uint64_t j) {
        const uint64_t li = si * a.P + j;
        PT_BOUND(a, si < a.nseeds && j < a.P);
        if (OUT) s_li[threadIdx.x] = li;
        uint64_t sid = a.seed_ids ? a.seed_ids[si] : si;
        if (sid > a.max_seed_id) {  // pid would overflow 64 bits: reported as PT_ERR_ARG
            atomicExch(a.stats + kStatBadId, 1ull);
            sid = 0;
        }
        x.pid = sid * a.P + j;
        x.sfix = smode ? (uint32_t)(j % a.S) : 0u;
        x.tmask = 0ull;
        x.sidx = (uint32_t)si;
        x.have_d0 = false;
        x.px = x.py = x.pz = 0.f;
        x.pxy = x.pzw = 0u;
        x.why = -1;
        if (UNQ) x.gen += 1u;
        if (begin(0u)) {
            x.alive = true;
        } else {
            // seed outside the volume (R12): finished right away (both halves), so the refill
            // loop may hand this lane another particle
            x.alive = false;
            write_outputs(0, kEndMask, x.qx, x.qy, x.qz);
            if (VB && H == 2u) {
                begin(1u);  // (outside again) point 0 of half 1's polyline
                write_outputs(0, kEndMask, x.qx, x.qy, x.qz);
            }
            particle_done();
        }
    };
    // commit a step (if c): new position, one visit of the new voxel (R13);
    // consecutive visits of the same voxel are merged (run length) and flushed with a
    // predicated RED when the voxel changes.  Straight-line except for the UNQ probe.
    // v: raster voxel, mk: map key (= v, or the record voxel with RVKEY)
    auto commit_if = [&](bool c, float nx_, float ny_, float nz_, uint32_t v, uint32_t mk) {
        // without outputs the position of an ended particle is never read again: no select
        x.qx = (c || !KEEPQ) ? nx_ : x.qx;
        x.qy = (c || !KEEPQ) ? ny_ : x.qy;
        x.qz = (c || !KEEPQ) ? nz_ : x.qz;
        x.n += c ? 1 : 0;
        if (UNQ) {
            unq_issue(c, v);
            const bool change = c && v != x.run_vox;
            x.prev_vox = change ? x.run_vox : x.prev_vox;
            x.run_vox = c ? v : x.run_vox;
        } else if (has_map) {
#if PT_RUNLEN
            const bool change = mk != x.run_vox;
            red_run(c && change && x.run_cnt != 0u, x.run_vox, x.run_cnt);
            x.run_cnt = c ? (change ? 1u : x.run_cnt + 1u) : x.run_cnt;
            x.run_vox = c ? mk : x.run_vox;
#else
            red_run(c, mk, 1u);  // ablation (iv): one global RED per committed step
#endif
        }
        if (OUT && a.conn && c) {  // NEXT-2: targets entered by committed steps (R21)
            PT_BOUND(a, v < a.V);
            const uint32_t lbl = __ldg(a.labels + v);
            x.tmask |= (lbl != 0u && lbl <= a.ntargets) ? (1ull << (lbl - 1u)) : 0ull;
        }
        if (OUT && a.o_paths && c && x.n < a.path_stride) {
            PT_BOUND(a, out_index() < a.out_n);
            float* pp = a.o_paths + (out_index() * (uint64_t)a.path_stride + (uint64_t)x.n) * 3u;
            pp[0] = __fadd_rn(x.qx, a.fcx);
            pp[1] = __fadd_rn(x.qy, a.fcy);
            pp[2] = __fadd_rn(x.qz, a.fcz);
        }
    };
    // Gather the record step nn will read at candidate position (cqx, cqy, cqz), nearest
    // voxel (ix, iy, iz) = v, sample s, if p; returns whether the candidate is outside the
    // mask (R11).  "Interpolation()": the nearest voxel (R2), or with PT_INTERP
    // the probabilistic neighbour (R23, stream 2 + half, block nn) with the nearest voxel
    // as fallback; the mask test is then the candidate's own mask byte.
    auto gather = [&](bool p, float cqx, float cqy, float cqz, uint32_t nrv, uint32_t v, uint32_t nn,
                      uint32_t s) -> bool {
        if (!interp) {
            if (p) PT_BOUND(a, (uint64_t)nrv * a.S + s < a.rec_n && s < a.S);
            ldg_record_if<RB>(p, rec_at(nrv, s), x.rv.w);
            return p && x.rv.outside();
        }
        const uint32_t hh = VB ? x.half : 0u;
        const uint4 I = philox(nn, 2u + hh);
        if (VN && nn == 0u && hh == 0u) x.winit = I.w;
        const int jx = interp_axis(cqx, a.cx, I.x), jy = interp_axis(cqy, a.cy, I.y), jz = interp_axis(cqz, a.cz, I.z);
        const bool jin = (unsigned)jx < (unsigned)a.nx && (unsigned)jy < (unsigned)a.ny && (unsigned)jz < (unsigned)a.nz;
        const uint32_t jv = ((uint32_t)jz * (uint32_t)a.ny + (uint32_t)jy) * (uint32_t)a.nx + (uint32_t)jx;
        if (p) PT_BOUND(a, (uint64_t)(jin ? recv(jx, jy, jz, jv) : nrv) * a.S + s < a.rec_n && s < a.S && v < a.V);
        ldg_record_if<RB>(p, rec_at(jin ? recv(jx, jy, jz, jv) : nrv, s), x.rv.w);
        const uint32_t mb = p ? (uint32_t)__ldg(a.mask + v) : 1u;
        const bool outside = p && mb == 0u;
        // the interpolated voxel lies outside the mask (sentinel record): the nearest voxel
        ldg_record_if<RB>(p && !outside && x.rv.outside(), rec_at(nrv, s), x.rv.w);
        return outside;
    };
    // R24: the fibre of the very first step, from the eligible fibres E = {j : f_j > fib_thr}
    auto initial_fibre = [&]() -> int {
        float fv[F];
        bool el[F];
        uint32_t ne = 0;
#pragma unroll
        for (int j = 0; j < F; ++j) {
            float ux, uy, uz;
            x.rv.fibre(j, ux, uy, uz, fv[j]);
            el[j] = fv[j] > a.fib_thr;
            ne += el[j] ? 1u : 0u;
        }
        if (ne == 0u) return 0;
        int js = 0;
        if (init_mode == 1u) {  // uniform over E: E[floor(w |E| / 2^32)]
            const uint32_t r = __umulhi(x.winit, ne);
            uint32_t before = 0;  // eligible fibres before j
#pragma unroll
            for (int j = 0; j < F; ++j) {
                js = (el[j] && before == r) ? j : js;
                before += el[j] ? 1u : 0u;
            }
        } else {  // f-weighted: first j in E with r < cumulative f (fp32, left to right)
            float tot = 0.f;
#pragma unroll
            for (int j = 0; j < F; ++j) tot = el[j] ? __fadd_rn(tot, fv[j]) : tot;
            const float r = __fmul_rn(__fmul_rn(__uint2float_rn(x.winit >> 8), 0x1p-24f), tot);
            float cum = 0.f;
            bool found = false;
            int last = 0;
#pragma unroll
            for (int j = 0; j < F; ++j) {
                if (el[j]) {
                    cum = __fadd_rn(cum, fv[j]);
                    if (!found && r < cum) {
                        js = j;
                        found = true;
                    }
                    last = j;
                }
            }
            if (!found) js = last;
        }
        return js;
    };
    // one step of Alg. 1's inner loop; k = position in the round
    auto step = [&](int k) {
        my_active += x.alive ? 1u : 0u;
        // a streamline's first step is always step 0 of a round (fresh particles start at a
        // round start; a live lane has n >= 1 after step 0): compile-time false for k > 0
        const bool first = k == 0 && x.n == 0 && (!VB || x.half == 0u);
        // choose the fibre closest to the previous direction: eligible iff
        // f_j > fib_thr (R7), strict >, lowest j wins (R8); the first step takes fibre 0
        // (R5; with R24 the round start moved the drawn fibre to slot 0).  "Interpolation()" of
        // Alg. 1 = this sample's record (R2).
        float vx, vy, vz, bc, best;
        bool neg;
        uint32_t dxy = 0u, dzw = 0u;  // fp16: the chosen direction, packed
        if constexpr (HALF) {
            // dot products on the packed halves (exact mixed-precision FMAs, see hdot)
            // R7 eligibility f_j > fib_thr: on the bench layouts (BL >= 0, launched only for
            // fib_thr >= 0) an integer compare of f's bits, in the high half of word 2j+1,
            // with those of the smallest binary16 above fib_thr (finite f, validated on load)
            auto elig = [&](uint32_t wzw) -> bool {
                return BL >= 0 ? (int32_t)wzw >= a.fib_h : half_hi(wzw) > a.fib_thr;
            };
            uint32_t cxy = x.rv.w[0], czw = x.rv.w[1];
            bc = hdot(cxy, czw, x.pxy, x.pzw);
            best = elig(czw) ? fabsf(bc) : -1.f;
#pragma unroll
            for (int j = 1; j < F; ++j) {
                const uint32_t uxy = x.rv.w[2 * j], uzw = x.rv.w[2 * j + 1];
                const float cj = hdot(uxy, uzw, x.pxy, x.pzw);
                const bool pick = !first && elig(uzw) && fabsf(cj) > best;
                best = pick ? fabsf(cj) : best;
                bc = pick ? cj : bc;
                cxy = pick ? uxy : cxy;
                czw = pick ? uzw : czw;
            }
            neg = first ? (x.W.w >> 31) != 0u : !(bc > 0.f);
            // sign * v: flip the sign bits (exact negation), then decode (exact)
            dxy = cxy ^ (neg ? 0x80008000u : 0u);
            dzw = (czw & 0xFFFFu) ^ (neg ? 0x8000u : 0u);
            vx = half_lo(dxy);
            vy = half_hi(dxy);
            vz = half_lo(dzw);
        } else {
            float f0;
            x.rv.fibre(0, vx, vy, vz, f0);
            bc = __fadd_rn(__fadd_rn(__fmul_rn(vx, x.px), __fmul_rn(vy, x.py)), __fmul_rn(vz, x.pz));
            best = f0 > a.fib_thr ? fabsf(bc) : -1.f;
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
            neg = first ? (x.W.w >> 31) != 0u : !(bc > 0.f);
        }
        // maximum angle, measured by the dot product (R4); orientation
        // kept (R9); first step: sign = top bit of word 3 of block 0 (R6, R16)
        const bool curv_ok = first || fabsf(bc) > a.curv_thr;
        // StepToNextPoint(): q' = q + h * (sign * v), no FMA (fp16: v already signed)
        const float dx = (HALF || !neg) ? vx : -vx, dy = (HALF || !neg) ? vy : -vy, dz = (HALF || !neg) ? vz : -vz;
        if (VB) {  // R22: half 0's first direction, defined even if the step is not committed
            const bool rec0 = first && x.alive;
            if constexpr (HALF) {
                x.d0xy = rec0 ? dxy : x.d0xy;
                x.d0zw = rec0 ? dzw : x.d0zw;
            }
            x.d0x = rec0 ? dx : x.d0x;
            x.d0y = rec0 ? dy : x.d0y;
            x.d0z = rec0 ? dz : x.d0z;
            x.have_d0 = x.have_d0 || rec0;
        }
        const float nqx = __fadd_rn(x.qx, __fmul_rn(a.step, dx));
        const float nqy = __fadd_rn(x.qy, __fmul_rn(a.step, dy));
        const float nqz = __fadd_rn(x.qz, __fmul_rn(a.step, dz));
        // NOB: coordinates in the margin-padded brick grid straight from the lookup; a
        // candidate outside the volume lands in a margin (or ragged) brick of sentinel records
        // and is rejected by its gather like any voxel outside the mask (R11)
        const int ix = axis_index(nqx, NOB ? a.pcx : a.cx), iy = axis_index(nqy, NOB ? a.pcy : a.cy),
                  iz = axis_index(nqz, NOB ? a.pcz : a.cz);
        const bool inb = NOB || ((unsigned)ix < (unsigned)a.nx && (unsigned)iy < (unsigned)a.ny && (unsigned)iz < (unsigned)a.nz);
        const uint32_t v = NOB ? 0u : ((uint32_t)iz * (uint32_t)a.ny + (uint32_t)iy) * (uint32_t)a.nx + (uint32_t)ix;
        const uint32_t crv = NOB ? recv_p((uint32_t)ix, (uint32_t)iy, (uint32_t)iz) : recv(ix, iy, iz, v);
        // stop criteria in order: maximum steps (R14), angle, volume (R11)
        const bool maxed = x.n == a.max_steps;
        const bool go = x.alive && !maxed && curv_ok && inb;
        // (without outputs the reason is never read: any value >= 0 marks "ended")
        x.why = (x.alive && !go) ? (!OUT ? kEndMask : maxed ? kEndMaxlen : (!curv_ok ? kEndCurv : kEndMask)) : x.why;
        x.alive = go;
        // (an ended particle's direction is never read)
        if constexpr (HALF) {
            x.pxy = (go || !KEEPQ) ? dxy : x.pxy;
            x.pzw = (go || !KEEPQ) ? dzw : x.pzw;
        } else {
            x.px = (go || !KEEPQ) ? dx : x.px;
            x.py = (go || !KEEPQ) ? dy : x.py;
            x.pz = (go || !KEEPQ) ? dz : x.pz;
        }
        if (k < kRoundSteps - 1) {
            if ((k + 1) % 3 == 0) {
                // the next step opens the round's next Philox block: a live lane has
                // committed t0 + k steps, so that block is (n + 1) / 3 (R16)
                x.W = philox(((uint32_t)x.n + 1u) / 3u, VB ? x.half : 0u);
            }
            const uint32_t w = ((k + 1) % 3 == 0) ? x.W.x : ((k + 1) % 3 == 1) ? x.W.y : x.W.z;
            const uint32_t sk = smode ? x.sfix : sample_of(w, a.S);
            const uint32_t nrv = crv;
            const bool outside = gather(go, nqx, nqy, nqz, nrv, v, (uint32_t)x.n + 1u, sk);
            x.why = outside ? kEndMask : x.why;
            x.alive = go && !outside;
            commit_if(x.alive, nqx, nqy, nqz, v, RVKEY ? nrv : v);
        } else {
            x.pend = go;  // next round's start gathers and tests it
            if (!RVKEY) x.gvox = go ? v : x.gvox;
            x.grv = go ? crv : x.grv;
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
        if (x.why >= 0) finish();  // particles (halves) that ended in the last round

        // ------------------------------------------------ lane refill (replaces the
        // paper's CPU Reduction()/segment relaunch)
        if (REFILL) {
            // refill once at least PT_REFILL_MIN lanes of the warp are free (or none is live)
            const uint32_t nfree = (uint32_t)__popc(__ballot_sync(kFull, !x.alive));
            if (!exhausted && nfree != 0u && (nfree >= (uint32_t)PT_REFILL_MIN || nfree == 32u)) {
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
        }
        if (!__any_sync(kFull, x.alive)) break;
        rounds += 1u;

        // ------------------------------------------------ round start: one Philox block,
        // gather of (pending candidate | seed) voxel = mask test + first step's record
        {
            const uint32_t t0 = (uint32_t)x.n + (x.pend ? 1u : 0u);  // a multiple of 3
            x.W = philox(t0 / 3u, VB ? x.half : 0u);
            const uint32_t s0 = smode ? x.sfix : sample_of(x.W.x, a.S);
            // the pending candidate, recomputed bit-identically from (q, d) instead of kept
            const float ppx = HALF ? half_lo(x.pxy) : x.px, ppy = HALF ? half_hi(x.pxy) : x.py,
                        ppz = HALF ? half_lo(x.pzw) : x.pz;
            const float cqx = x.pend ? __fadd_rn(x.qx, __fmul_rn(a.step, ppx)) : x.qx;
            const float cqy = x.pend ? __fadd_rn(x.qy, __fmul_rn(a.step, ppy)) : x.qy;
            const float cqz = x.pend ? __fadd_rn(x.qz, __fmul_rn(a.step, ppz)) : x.qz;
            if (VN && init_mode != 0u && !interp && t0 == 0u && (!VB || x.half == 0u) && x.alive)
                x.winit = philox(0u, 2u).w;  // R24 draw (with PT_INTERP the gather computes it)
            // seed outside the mask (R12) or pending candidate rejected (R11)
            const bool outside = gather(x.alive, cqx, cqy, cqz, x.grv, x.gvox, t0, s0);
            x.why = outside ? kEndMask : x.why;
            x.alive = x.alive && !outside;
            commit_if(x.pend && !outside, cqx, cqy, cqz, x.gvox, RVKEY ? x.grv : x.gvox);
            // R24: the first step of half 0 takes the drawn fibre: move it to slot 0 of the
            // record (the first step uses only the chosen fibre's vector)
            if (VN && F > 1 && init_mode != 0u) {
                const bool fresh = x.alive && t0 == 0u && (!VB || x.half == 0u);
                if (__any_sync(kFull, fresh)) {
                    const int js = fresh ? initial_fibre() : 0;
                    x.rv.swap_to_front(js);
                }
            }
            x.pend = false;
        }

        // ------------------------------------------------ the round's steps
#pragma unroll
        for (int k = 0; k < kRoundSteps; ++k) step(k);
    }

    // ---- counters: one atomic per warp (64-bit sums of the per-lane counters)
    unsigned long long s_steps = my_steps, s_parts = my_particles, s_act = my_active, s_uq = my_unique;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        s_steps += __shfl_xor_sync(kFull, s_steps, o);
        s_parts += __shfl_xor_sync(kFull, s_parts, o);
        s_act += __shfl_xor_sync(kFull, s_act, o);
        if (UNQ) s_uq += __shfl_xor_sync(kFull, s_uq, o);
    }
    if (lane == 0) {
        atomicAdd(a.stats + kStatSteps, s_steps);
        atomicAdd(a.stats + kStatParticles, s_parts);
        atomicAdd(a.stats + kStatLaneActive, s_act);
        atomicAdd(a.stats + kStatLaneSlots, (unsigned long long)rounds * (unsigned long long)kRoundSteps * 32ull);
        if (UNQ) atomicAdd(a.stats + kStatUnique, s_uq);
    }
}

// grid of one launch: persistent (at most #SMs x resident CTAs, or fewer when the job or the
// UNQ hash sets are smaller) or one thread per particle
template <int F, bool HALF, bool REFILL, bool OUT, int BL, int VM, bool UNQ, bool NB = false>
cudaError_t launch_track_kernel(const TrackArgs& a, int num_sms, cudaStream_t st) {
    auto k = track_kernel<F, HALF, REFILL, OUT, BL, VM, UNQ, NB>;
    constexpr int TPB = track_tpb<REFILL, VM, UNQ>();
    if (a.nparticles == 0) return cudaSuccess;
    unsigned grid;
    if (REFILL) {
        int per_sm = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, TPB, 0);
        if (e != cudaSuccess) return e;
        if (per_sm < 1) return cudaErrorInvalidConfiguration;
        const uint64_t need = (a.nparticles + (uint64_t)TPB - 1) / (uint64_t)TPB;
        uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
        if (UNQ && a.max_ctas < full) full = a.max_ctas;
        grid = (unsigned)(need < full ? need : full);
    } else {
        grid = (unsigned)((a.nparticles + TPB - 1) / TPB);
    }
    k<<<grid, TPB, 0, st>>>(a);
    return cudaGetLastError();
}

// All instantiations for one (F, HALF); pt_track_f<F>_<h|f>.cu define launch_track_f<F>.
template <int F, bool HALF, int VM>
cudaError_t launch_track_var(const TrackArgs& a, const TrackMode& m, int num_sms, cudaStream_t st) {
    return m.out ? launch_track_kernel<F, HALF, true, true, -1, VM, false>(a, num_sms, st)
                 : launch_track_kernel<F, HALF, true, false, -1, VM, false>(a, num_sms, st);
}

template <int F, bool HALF>
cudaError_t launch_track_fh(const TrackArgs& a, const TrackMode& m, int num_sms, cudaStream_t st) {
    if (m.simple) {  // ablation (i): default semantics only
        return m.out ? launch_track_kernel<F, HALF, false, true, -1, 0, false>(a, num_sms, st)
                     : launch_track_kernel<F, HALF, false, false, -1, 0, false>(a, num_sms, st);
    }
    if (m.unique) {  // NEXT-2: default semantics, or every variant switched at run time
        if (m.var)
            return m.out ? launch_track_kernel<F, HALF, true, true, -1, kVarAll, true>(a, num_sms, st)
                         : launch_track_kernel<F, HALF, true, false, -1, kVarAll, true>(a, num_sms, st);
        return m.out ? launch_track_kernel<F, HALF, true, true, -1, 0, true>(a, num_sms, st)
                     : launch_track_kernel<F, HALF, true, false, -1, 0, true>(a, num_sms, st);
    }
    if (m.var) {  // the compiled-in variants are exactly the requested ones (forced: all)
        const int vm = (a.bidir ? kVarBidir : 0) | (a.interp ? kVarInterp : 0) | (a.init_mode ? kVarInit : 0);
        switch (vm) {
            case 1: return launch_track_var<F, HALF, 1>(a, m, num_sms, st);
            case 2: return launch_track_var<F, HALF, 2>(a, m, num_sms, st);
            case 3: return launch_track_var<F, HALF, 3>(a, m, num_sms, st);
            case 4: return launch_track_var<F, HALF, 4>(a, m, num_sms, st);
            case 5: return launch_track_var<F, HALF, 5>(a, m, num_sms, st);
            case 6: return launch_track_var<F, HALF, 6>(a, m, num_sms, st);
            default: return launch_track_var<F, HALF, kVarAll>(a, m, num_sms, st);  // 7, or PT_KERNEL_VARIANT alone
        }
    }
    if (m.out) return launch_track_kernel<F, HALF, true, true, -1, 0, false>(a, num_sms, st);
    if (a.sample_mode) return launch_track_kernel<F, HALF, true, false, -1, 0, false>(a, num_sms, st);
    // the bench path: record layout as a compile-time constant, random sample per step
    // (the compile-time layouts compare fp16 f bits as integers: fib_thr >= 0 only)
    // (track_rv_keys: exactly the kBrickLog instantiation keys the map by record voxel)
    if (track_rv_keys(a, m, HALF)) {  // with margin bricks covering every candidate: no bounds test
        if (PT_REC_MARGIN && a.nobounds)
            return launch_track_kernel<F, HALF, true, false, (int)kBrickLog, 0, false, true>(a, num_sms, st);
        return launch_track_kernel<F, HALF, true, false, (int)kBrickLog, 0, false>(a, num_sms, st);
    }
    if (HALF && !(a.fib_thr >= 0.f)) return launch_track_kernel<F, HALF, true, false, -1, 0, false>(a, num_sms, st);
    if (a.rb_log == 0) return launch_track_kernel<F, HALF, true, false, 0, 0, false>(a, num_sms, st);
    if (a.rb_log == kBrickLog) return launch_track_kernel<F, HALF, true, false, (int)kBrickLog, 0, false>(a, num_sms, st);
    return cudaErrorInvalidValue;
}

}  // namespace pt
