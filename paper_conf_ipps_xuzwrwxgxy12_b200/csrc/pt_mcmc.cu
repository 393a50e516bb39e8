// pt_mcmc.cu -- NEXT-4: Metropolis-Hastings sampling of the multiple partial volume model
// (Eq. 1; Sec. IV-A and Fig. 2) on sm_100a, binary64 (reading M4).
//
// The paper runs one thread per voxel.  Here a group of LPV lanes owns a voxel (two
// voxels per warp, 16 lanes each, for n <= 64; one voxel per warp above) and lane l of a
// group holds measurements l, l + LPV, ...: the per-measurement terms of Eq. 1 stay in
// registers for the whole chain (e^{-b d}, e^{-b d (r.v_j)^2}, r.v_j), so a proposal of S0,
// sigma or f_j costs no exponential, an angle proposal one per measurement and a d proposal
// N per measurement plus one per b-shell; the sum of squared residuals is a group
// reduction.  Lane k of a group owns parameter k (value, proposal width, counters, sin/cos).
// The draws are counter-based (M6) and omega'_k only depends on omega_k, which no other MH
// step of the loop changes: the lanes compute the Box-Muller draws of several loops at
// once, lane k forms candidate k and its transcendental by-products (ln sigma', sincos,
// ln|sin theta'|) at the loop's start, and step k only broadcasts them from lane k.
//
// Results follow contract C-MCMC of DESIGN.md §12 in the oracle's operation order; the
// oracle uses glibc's exp/log/sin/cos, this file CUDA's (both within an ulp or two), the
// residual sum is a lane tree instead of a sequential loop and a*b+c is fused into a DFMA,
// so samples agree to ~1e-13 relative rather than bit for bit (the parity bar of DESIGN.md
// §12).
#include <cuda_runtime.h>
#include <cub/device/device_select.cuh>
#include <thrust/iterator/counting_iterator.h>

#include <cstdint>

#include "pt_device.cuh"
#include "pt_internal.h"

namespace pt {

namespace {

constexpr uint32_t kTag = 0x4D434D43u;  // "MCMC": Philox counter word 3 (M6)
constexpr double kTwoPi = 6.283185307179586;
constexpr int kMcmcThreads = 128;         // 4 warps per CTA
constexpr int kMaxShells = 8;             // distinct b-values handled with one exp each
#ifndef PT_MCMC_VPW
#define PT_MCMC_VPW 2  // voxels per warp for nmeas <= 64 (1: one voxel per warp always)
#endif
#ifndef PT_MCMC_MIN_BLOCKS
#define PT_MCMC_MIN_BLOCKS 3  // CTAs per SM the register budget must allow (12 warps; 4 spills: -1.3 %, r02u)
#endif

#ifndef PT_MCMC_FMA
#define PT_MCMC_FMA 1  // contract a*b+c into DFMA in the per-measurement terms
#endif
// a * b + c: one fused DFMA (PT_MCMC_FMA) or a rounded product and a rounded sum (the
// oracle's order; the library is built with -fmad=false, so only this helper fuses)
__device__ __forceinline__ double madd(double a, double b, double c) {
#if PT_MCMC_FMA
    return __fma_rn(a, b, c);
#else
    return a * b + c;
#endif
}

// Sum over the LPV lanes of a voxel group (xor butterfly), then the group's first lane's
// value for every lane of the group (the butterfly's lanes may differ in the last bit).
template <int LPV>
__device__ __forceinline__ double group_sum(double v) {
#pragma unroll
    for (int o = LPV / 2; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o, LPV);
    return __shfl_sync(kFull, v, 0, LPV);
}

// VPW voxels per warp, LPV = 32 / VPW lanes per voxel, MPL measurements per lane.
// FULL: n == LPV * MPL (every measurement slot holds a measurement; no masking).
template <int N, int MPL, int VPW, bool FULL>
__global__ void __launch_bounds__(kMcmcThreads, PT_MCMC_MIN_BLOCKS) mcmc_kernel(const __grid_constant__ McmcArgs a) {
    constexpr int NP = 3 + 3 * N;
    constexpr int LPV = 32 / VPW;
    static_assert(NP <= LPV, "a lane per parameter");
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t gl = lane % (uint32_t)LPV;   // lane within the voxel group
    const uint32_t grp = lane / (uint32_t)LPV;  // voxel group within the warp
    const int n = a.nmeas;
    const double np1 = (double)(n + 1);

    // the gradient table (b, r) is the same for every voxel: shared memory, SoA (a lane
    // reads entry gl + LPV m: distinct banks within a group, broadcast across groups);
    // entries >= n are zero.  Measurement i of the voxel: i = gl + LPV m.
    __shared__ float s_b[LPV * MPL], s_rx[LPV * MPL], s_ry[LPV * MPL], s_rz[LPV * MPL];
    // the same in binary64 for the hot loops (no float->double conversion per use)
    __shared__ double s_bd[LPV * MPL], s_rxd[LPV * MPL], s_ryd[LPV * MPL], s_rzd[LPV * MPL];
    // each lane's measurements of its voxel in binary64 (lane-private slots)
    __shared__ double s_y[kMcmcThreads / 32][MPL][32];
    // the distinct b-values ("shells", <= kMaxShells) and each measurement's shell: a d
    // proposal then needs one e^{-b d'} per shell instead of one per measurement
    __shared__ float s_shell[kMaxShells];
    __shared__ int s_sidx[LPV * MPL];
    __shared__ int s_nshell;
    for (int i = threadIdx.x; i < LPV * MPL; i += blockDim.x) {
        const bool in = i < n;
        s_b[i] = in ? a.bvals[i] : 0.f;
        s_rx[i] = in ? a.bvecs[3 * i] : 0.f;
        s_ry[i] = in ? a.bvecs[3 * i + 1] : 0.f;
        s_rz[i] = in ? a.bvecs[3 * i + 2] : 0.f;
        s_bd[i] = (double)s_b[i];
        s_rxd[i] = (double)s_rx[i];
        s_ryd[i] = (double)s_ry[i];
        s_rzd[i] = (double)s_rz[i];
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int ns = 0;
        for (int i = 0; i < LPV * MPL; ++i) {
            int u = 0;
            while (u < ns && s_shell[u] != s_b[i]) ++u;
            if (u == ns) {
                if (ns == kMaxShells) {
                    ns = 0;  // too many shells: per-measurement exponentials
                    break;
                }
                s_shell[ns++] = s_b[i];
            }
            s_sidx[i] = u;
        }
        s_nshell = ns;
    }
    __syncthreads();
    const int nshell = s_nshell;
#define BF(m) s_b[gl + LPV * (m)]
#define RX(m) s_rx[gl + LPV * (m)]
#define RY(m) s_ry[gl + LPV * (m)]
#define RZ(m) s_rz[gl + LPV * (m)]
#define BD(m) s_bd[gl + LPV * (m)]
#define RXD(m) s_rxd[gl + LPV * (m)]
#define RYD(m) s_ryd[gl + LPV * (m)]
#define RZD(m) s_rzd[gl + LPV * (m)]
#define YD(m) s_y[threadIdx.x >> 5][m][lane]
    bool valid[MPL];
    float yf[MPL];
#pragma unroll
    for (int m = 0; m < MPL; ++m) valid[m] = FULL || (int)gl + LPV * m < n;
    unsigned long long acc_tot = 0ull;

    for (;;) {
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(a.queue, (uint32_t)VPW);
        base = __shfl_sync(kFull, base, 0);
        if (base >= a.nvox) break;
        const uint32_t slot = base + grp;
        const bool gact = slot < a.nvox;  // a group without a voxel computes on base's, writes nothing
        const uint32_t v = a.vox[gact ? slot : base];
        const uint64_t V = a.V;
#if PT_CHECK_BOUNDS
        bool bad = !(v < V) || (gact && !(slot < a.nvox));
        for (int m = 0; m < MPL; ++m) bad = bad || (valid[m] && !((int)gl + LPV * m < a.nmeas));
        if (bad) atomicOr(a.stats + kMcmcStatBadAccess, 1ull);
#endif
#pragma unroll
        for (int m = 0; m < MPL; ++m) {
            yf[m] = valid[m] ? a.dwi[(uint64_t)(gl + LPV * m) * V + v] : 0.f;
            YD(m) = (double)yf[m];
        }

        double w[NP];
        double sth[N], cth[N], sph[N], cph[N], lsin[N];
        // ------------------------------------------------ initial state (M7 or given)
        if (a.init) {
#pragma unroll
            for (int k = 0; k < NP; ++k) w[k] = a.init[(uint64_t)k * V + v];
        } else {
            double s0 = 0.0, sd = 0.0, bsum = 0.0, ymax = -__longlong_as_double(0x7FF0000000000000ll);
            int c0 = 0, cd = 0;
#pragma unroll
            for (int m = 0; m < MPL; ++m) {
                if (!valid[m]) continue;
                const double y = (double)yf[m];
                ymax = y > ymax ? y : ymax;
                if (BF(m) == 0.f) {
                    s0 += y;
                    c0 += 1;
                } else {
                    sd += y;
                    bsum += (double)BF(m);
                    cd += 1;
                }
            }
            s0 = group_sum<LPV>(s0);
            sd = group_sum<LPV>(sd);
            bsum = group_sum<LPV>(bsum);
#pragma unroll
            for (int o = LPV / 2; o > 0; o >>= 1) {
                c0 += __shfl_xor_sync(kFull, c0, o, LPV);
                cd += __shfl_xor_sync(kFull, cd, o, LPV);
                ymax = fmax(ymax, __shfl_xor_sync(kFull, ymax, o, LPV));
            }
            double S0 = c0 ? s0 / (double)c0 : ymax;
            if (!(S0 > 0.0)) S0 = 1.0;
            double d = 0.0;
            if (cd) d = -log((sd / (double)cd) / S0) / (bsum / (double)cd);
            if (!(d > 0.0) || !isfinite(d)) d = cd ? 1.0 / (bsum / (double)cd) : 1.0;
            w[0] = S0;
            w[1] = d;
            // fibre j: DW direction of the smallest signal with |r.v_k| < 1/2 for earlier fibres
            float px[N], py[N], pz[N];
            bool have[N];
#pragma unroll
            for (int j = 0; j < N; ++j) {
                float by = __int_as_float(0x7F800000);
                int bi = 0x7FFFFFFF;
#pragma unroll
                for (int m = 0; m < MPL; ++m) {
                    bool ok = valid[m] && BF(m) != 0.f;
#pragma unroll
                    for (int k = 0; k < j; ++k) {
                        const double dot = ((double)RX(m) * (double)px[k] + (double)RY(m) * (double)py[k]) +
                                           (double)RZ(m) * (double)pz[k];
                        if (have[k]) ok = ok && fabs(dot) < 0.5;  // a missing pick constrains nothing
                    }
                    const int i = (int)gl + LPV * m;
                    if (ok && (yf[m] < by || (yf[m] == by && i < bi))) {
                        by = yf[m];
                        bi = i;
                    }
                }
#pragma unroll
                for (int o = LPV / 2; o > 0; o >>= 1) {
                    const float oy = __shfl_xor_sync(kFull, by, o, LPV);
                    const int oi = __shfl_xor_sync(kFull, bi, o, LPV);
                    if (oy < by || (oy == by && oi < bi)) {
                        by = oy;
                        bi = oi;
                    }
                }
                have[j] = bi != 0x7FFFFFFF;
                px[j] = py[j] = pz[j] = 0.f;
                if (have[j]) {
                    px[j] = a.bvecs[3 * bi];
                    py[j] = a.bvecs[3 * bi + 1];
                    pz[j] = a.bvecs[3 * bi + 2];
                }
                w[3 + 3 * j] = j == 0 ? 0.3 : 0.1;
                if (have[j]) {
                    const double z = (double)pz[j];
                    w[4 + 3 * j] = acos(z < -1.0 ? -1.0 : (z > 1.0 ? 1.0 : z));
                    w[5 + 3 * j] = atan2((double)py[j], (double)px[j]);
                } else if (j == 0) {
                    w[4] = 1.0;
                    w[5] = 0.0;
                } else {
                    w[4 + 3 * j] = w[4] + (j == 1 ? 1.5707963267948966 : 0.0);
                    w[5 + 3 * j] = w[5] + (j == 2 ? 1.5707963267948966 : 0.0);
                }
            }
            w[2] = 1.0;  // sigma: set below from the initial model's residual
        }
#pragma unroll
        for (int j = 0; j < N; ++j) {
            sincos(w[4 + 3 * j], &sth[j], &cth[j]);
            sincos(w[5 + 3 * j], &sph[j], &cph[j]);
            lsin[j] = log(fabs(sth[j]));
        }

        // ------------------------------------------------ per-measurement caches (Eq. 1)
        double e0[MPL], ej[N][MPL], dj[N][MPL];
        double fj[N];
        double sumf = 0.0;
#pragma unroll
        for (int j = 0; j < N; ++j) {
            fj[j] = w[3 + 3 * j];
            sumf = sumf + fj[j];
        }
        double sse = 0.0;
#pragma unroll
        for (int m = 0; m < MPL; ++m) {
            const double b = BD(m);
            const double bd = b * w[1];
            e0[m] = exp(-bd);
            double acc = (1.0 - sumf) * e0[m];
#pragma unroll
            for (int j = 0; j < N; ++j) {
                const double vx = sth[j] * cph[j], vy = sth[j] * sph[j], vz = cth[j];
                dj[j][m] = madd(RZD(m), vz, madd(RYD(m), vy, RXD(m) * vx));
                ej[j][m] = exp(-(bd * (dj[j][m] * dj[j][m])));
                acc = madd(fj[j], ej[j][m], acc);
            }
            const double r = YD(m) - w[0] * acc;
            sse = valid[m] ? madd(r, r, sse) : sse;
        }
        sse = group_sum<LPV>(sse);
        if (!a.init) {
            double sig = sqrt(sse / (double)n);
            if (!(sig >= 1e-3 * w[0])) sig = 1e-3 * w[0];
            w[2] = sig;
        }
        // uniform copies of the parameters the likelihood needs every step
        double S0 = w[0], dd = w[1], sig = w[2];
        double lsig = log(sig);
        double inv2s2 = 1.0 / (2.0 * sig * sig);  // 1 / (2 sigma^2), refreshed when sigma moves
        double lp = -np1 * lsig - sse * inv2s2;
#pragma unroll
        for (int j = 0; j < N; ++j) lp = lp + lsin[j];

        // ------------------------------------------------ lane k owns parameter k: its value,
        // proposal width (M8), acceptance counters and, for angles, sin / cos (/ ln|sin|)
        double my_w = w[0];
#pragma unroll
        for (int k = 1; k < NP; ++k) my_w = gl == (uint32_t)k ? w[k] : my_w;
        double my_prop = 0.1;
        if (gl == 0u) my_prop = 0.01 * S0;
        else if (gl == 1u) my_prop = 0.1 * dd;
        else if (gl == 2u) my_prop = 0.1 * sig;
        else if (gl >= 3u && (gl - 3u) % 3u == 0u) my_prop = 0.05;
        double my_s = 0.0, my_c = 0.0;  // angle lanes: sin, cos of the current value
#pragma unroll
        for (int j = 0; j < N; ++j) {
            if (gl == (uint32_t)(4 + 3 * j)) {
                my_s = sth[j];
                my_c = cth[j];
            } else if (gl == (uint32_t)(5 + 3 * j)) {
                my_s = sph[j];
                my_c = cph[j];
            }
        }
        uint32_t my_acc = 0u, my_rej = 0u, my_tot = 0u;
        double bz = 0.0, blu = 0.0;  // batched draws (lanes < B * NP)

        const uint32_t loops = a.loops;
        for (uint32_t t = 0; t < loops; ++t) {
            // The draws (M6) do not depend on the state: every B = 32 / NP loops, lane
            // i*NP + k computes draw k of loop t + i (up to 32 draws per batch).
            constexpr int B = LPV / NP;
            const uint32_t ph = t % (uint32_t)B;
            if (ph == 0u && gl < (uint32_t)(B * NP)) {
                const uint32_t tt = t + gl / (uint32_t)NP, kk = gl % (uint32_t)NP;
                const uint4 R = philox4x32_10(make_uint4(tt, v, kk, kTag), a.key0, a.key1);
                const double u1 = ((double)R.x + 0.5) * 0x1p-32;
                const double u2 = (double)R.y * 0x1p-32;
                const double u3 = ((double)R.z + 0.5) * 0x1p-32;
                bz = sqrt(-2.0 * log(u1)) * cos(kTwoPi * u2);
                blu = log(u3);
            }
            // lane k < NP: draw k of this loop, candidate omega'_k and its by-products
            const uint32_t src = ph * (uint32_t)NP + (gl < (uint32_t)NP ? gl : 0u);
            const double z = __shfl_sync(kFull, bz, src, LPV);
            const double clu = __shfl_sync(kFull, blu, src, LPV);
            // branch-free by-products (one sincos and one log per lane instead of a
            // divergent branch per parameter kind): sigma lane: ca = ln sigma'; theta lanes:
            // (sin, cos, ln|sin|); phi lanes: (sin, cos); the others' values are unused
            const double cz = my_w + my_prop * z;
            double sn, cs;
            sincos(gl >= 3u ? cz : 0.0, &sn, &cs);
            const double lx = log(gl == 2u ? cz : fabs(sn));
            const double ca = gl == 2u ? lx : sn, cb = cs, cc = lx;
            // Fig. 2: the MH step, repeated NumParameters times
#pragma unroll
            for (int k = 0; k < NP; ++k) {
                if (a.fixed & (1u << k)) continue;
                const double cand = __shfl_sync(kFull, cz, k, LPV);
                const double lu = __shfl_sync(kFull, clu, k, LPV);
                const int jf = k >= 3 ? (k - 3) / 3 : 0;       // fibre of an f/theta/phi step
                const int r3 = k >= 3 ? (k - 3) % 3 : -1;      // 0 f, 1 theta, 2 phi
                // support (M3)
                bool ok;
                double nsumf = sumf;
                if (k < 3) {
                    ok = cand > 0.0;
                } else if (r3 == 0) {
                    nsumf = 0.0;
#pragma unroll
                    for (int j = 0; j < N; ++j) nsumf = nsumf + (j == jf ? cand : fj[j]);
                    ok = cand >= 0.0 && nsumf <= 1.0;
                } else {
                    ok = true;
                }
                // (no early exit: the groups of a warp may disagree; a candidate outside the
                // support is evaluated and then rejected through `ok`)
                double xa = 0.0, xb = 0.0, xc = 0.0;  // the candidate's by-products (lane k)
                double nvx = 0.0, nvy = 0.0, nvz = 0.0;
                if (k == 2) {
                    xa = __shfl_sync(kFull, ca, k, LPV);
                } else if (r3 == 1 || r3 == 2) {
                    xa = __shfl_sync(kFull, ca, k, LPV);
                    xb = __shfl_sync(kFull, cb, k, LPV);
                    // the fibre's other angle, current value, from its owner lane
                    const int other = r3 == 1 ? k + 1 : k - 1;
                    const double os = __shfl_sync(kFull, my_s, other, LPV);
                    const double oc = __shfl_sync(kFull, my_c, other, LPV);
                    if (r3 == 1) {  // theta' with the current phi
                        xc = __shfl_sync(kFull, cc, k, LPV);
                        nvx = xa * oc;
                        nvy = xa * os;
                        nvz = xb;
                    } else {        // phi' with the current theta
                        nvx = os * xb;
                        nvy = os * xa;
                        nvz = oc;
                    }
                }
                double nsse = 0.0, nlp;
                double ne[MPL], nd[MPL], nej[N][MPL];
                double eshell = 0.0;
                if (k == 1 && nshell)  // same operations as the per-measurement e^{-b d'}
                    eshell = exp(-((double)s_shell[gl < (uint32_t)nshell ? gl : 0u] * cand));
                double ninv = inv2s2;
                if (k == 2) {
                    ninv = 1.0 / (2.0 * cand * cand);
                    nlp = -np1 * xa - sse * ninv;
#pragma unroll
                    for (int j = 0; j < N; ++j) nlp = nlp + lsin[j];
                } else {
#pragma unroll
                    for (int m = 0; m < MPL; ++m) {
                        double mu;
                        if (k == 0) {  // the mixture is recomputed (3 DP ops) instead of cached
                            double accm = (1.0 - sumf) * e0[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) accm = madd(fj[j], ej[j][m], accm);
                            mu = cand * accm;
                        } else if (k == 1) {
                            const double bd = BD(m) * cand;
                            if (nshell) {  // e^{-b d'} of this measurement's shell (lane u: shell u)
                                ne[m] = __shfl_sync(kFull, eshell, s_sidx[gl + LPV * m], LPV);
                            } else {
                                ne[m] = exp(-bd);
                            }
                            double accm = (1.0 - sumf) * ne[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) {
                                nej[j][m] = exp(-(bd * (dj[j][m] * dj[j][m])));
                                accm = madd(fj[j], nej[j][m], accm);
                            }
                            mu = S0 * accm;
                        } else if (r3 == 0) {
                            double accm = (1.0 - nsumf) * e0[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) accm = madd(j == jf ? cand : fj[j], ej[j][m], accm);
                            mu = S0 * accm;
                        } else {
                            const double bd = BD(m) * dd;
                            nd[m] = madd(RZD(m), nvz, madd(RYD(m), nvy, RXD(m) * nvx));
                            ne[m] = exp(-(bd * (nd[m] * nd[m])));
                            double accm = (1.0 - sumf) * e0[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) accm = madd(fj[j], j == jf ? ne[m] : ej[j][m], accm);
                            mu = S0 * accm;
                        }
                        const double r = YD(m) - mu;
                        nsse = valid[m] ? madd(r, r, nsse) : nsse;
                    }
                    nsse = group_sum<LPV>(nsse);
                    nlp = -np1 * lsig - nsse * inv2s2;
#pragma unroll
                    for (int j = 0; j < N; ++j) nlp = nlp + ((r3 == 1 && j == jf) ? xc : lsin[j]);
                }
                // accept with probability min(r, 1): ln u < lp' - lp
                const bool accept = ok && lu < nlp - lp;
                if (gl == (uint32_t)k) {
                    my_acc += accept ? 1u : 0u;
                    my_tot += accept ? 1u : 0u;
                    my_rej += accept ? 0u : 1u;
                    if (accept) {
                        my_w = cz;
                        my_s = ca;
                        my_c = cb;
                    }
                }
                if (accept) {
                    lp = nlp;
                    if (k == 0) {
                        S0 = cand;
                        sse = nsse;
                    } else if (k == 1) {
                        dd = cand;
                        sse = nsse;
#pragma unroll
                        for (int m = 0; m < MPL; ++m) {
                            e0[m] = ne[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) ej[j][m] = nej[j][m];
                        }
                    } else if (k == 2) {
                        sig = cand;
                        lsig = xa;
                        inv2s2 = ninv;
                    } else {
                        sse = nsse;
                        if (r3 == 0) {
                            fj[jf] = cand;
                            sumf = nsumf;
                        } else if (r3 == 1) {
                            lsin[jf] = xc;
                        }
#pragma unroll
                        for (int m = 0; m < MPL; ++m) {
                            if (r3 != 0) {
                                dj[jf][m] = nd[m];
                                ej[jf][m] = ne[m];
                            }
                        }
                    }
                }
            }
            // Fig. 2: every K loops the acceptance rates update the proposals (M8); lane k
            // updates its own parameter's width
            if ((t + 1u) % a.adapt_every == 0u) {
                my_prop = my_prop * sqrt((5.0 * (double)(my_acc + 1u)) / (3.0 * (double)(my_rej + 1u)));
                my_acc = my_rej = 0u;
            }
            // samples after the burn-in, every L loops; lane k writes omega_k
            if (t >= a.burnin && (t - a.burnin + 1u) % a.interval == 0u) {
                const uint32_t s = (t - a.burnin + 1u) / a.interval - 1u;
#if PT_CHECK_BOUNDS
                if (s >= a.nsamples) atomicOr(a.stats + kMcmcStatBadAccess, 1ull);
#endif
                if (gact && gl < (uint32_t)NP) a.samples[((uint64_t)gl * a.nsamples + s) * V + v] = my_w;
            }
        }
        if (a.accepted && gact && gl < (uint32_t)NP) a.accepted[(uint64_t)gl * V + v] = my_tot;
        if (gact && gl < (uint32_t)NP) acc_tot += my_tot;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc_tot += __shfl_xor_sync(kFull, acc_tot, o);
    if (lane == 0 && acc_tot) atomicAdd(a.stats + kMcmcStatAccepted, acc_tot);
#undef BF
#undef RX
#undef RY
#undef RZ
#undef BD
#undef RXD
#undef RYD
#undef RZD
#undef YD
}

template <int N, int MPL, int VPW>
cudaError_t launch_m(const McmcArgs& a, int num_sms, cudaStream_t st) {
    constexpr int LPV = 32 / VPW;
    auto k = a.nmeas == LPV * MPL ? mcmc_kernel<N, MPL, VPW, true> : mcmc_kernel<N, MPL, VPW, false>;
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kMcmcThreads, 0);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    const uint64_t per_cta = (uint64_t)(kMcmcThreads / 32) * VPW;  // voxels in flight per CTA
    const uint64_t need = ((uint64_t)a.nvox + per_cta - 1) / per_cta;
    const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
    const uint64_t grid = need < full ? need : full;
    if (grid == 0) return cudaSuccess;
    k<<<(unsigned)grid, kMcmcThreads, 0, st>>>(a);
    return cudaGetLastError();
}

template <int N>
cudaError_t launch_mn(const McmcArgs& a, int num_sms, cudaStream_t st) {
    // up to 64 measurements: two voxels per warp (16 lanes each, <= 4 measurements per lane),
    // which halves the per-voxel cost of the serial part of an MH step (reduction, decision)
    if (PT_MCMC_VPW == 2 && a.nmeas <= 64) {
        switch ((a.nmeas + 15) / 16) {
            case 1: return launch_m<N, 1, 2>(a, num_sms, st);
            case 2: return launch_m<N, 2, 2>(a, num_sms, st);
            case 3: return launch_m<N, 3, 2>(a, num_sms, st);
            case 4: return launch_m<N, 4, 2>(a, num_sms, st);
            default: return cudaErrorInvalidValue;
        }
    }
    switch ((a.nmeas + 31) / 32) {
        case 1: return launch_m<N, 1, 1>(a, num_sms, st);
        case 2: return launch_m<N, 2, 1>(a, num_sms, st);
        case 3: return launch_m<N, 3, 1>(a, num_sms, st);
        case 4: return launch_m<N, 4, 1>(a, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

__global__ void mask_flags_kernel(const uint8_t* __restrict__ mask, uint64_t V, uint8_t* __restrict__ flags) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += (uint64_t)gridDim.x * blockDim.x)
        flags[i] = mask[i] != 0 ? 1 : 0;
}

// (theta, phi) -> unit vector, f -> float (R20: the conversion is outside the trackers)
__global__ void samples_to_volume_kernel(const double* __restrict__ smp, const uint8_t* __restrict__ mask,
                                         uint64_t V, int N, int S, float* __restrict__ dyads, float* __restrict__ f) {
    const uint64_t total = (uint64_t)N * S * V;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t v = i % V;
        const uint64_t js = i / V;          // j * S + s
        const uint64_t j = js / S, s = js - j * S;
        float x = 0.f, y = 0.f, z = 0.f, ff = 0.f;
        if (mask[v]) {
            const double fj = smp[((3 + 3 * j) * S + s) * V + v];
            const double th = smp[((4 + 3 * j) * S + s) * V + v];
            const double ph = smp[((5 + 3 * j) * S + s) * V + v];
            double st, ct, sp, cp;
            sincos(th, &st, &ct);
            sincos(ph, &sp, &cp);
            x = (float)(st * cp);
            y = (float)(st * sp);
            z = (float)ct;
            ff = (float)fj;
        }
        dyads[3 * i] = x;
        dyads[3 * i + 1] = y;
        dyads[3 * i + 2] = z;
        f[i] = ff;
    }
}

}  // namespace

size_t mcmc_select_temp_bytes(uint64_t V) {
    size_t bytes = 0;
    cub::DeviceSelect::Flagged(nullptr, bytes, thrust::counting_iterator<uint32_t>(0), (const uint8_t*)nullptr,
                               (uint32_t*)nullptr, (uint32_t*)nullptr, (int64_t)V);
    return bytes;
}

cudaError_t launch_mcmc_voxel_list(const uint8_t* mask, uint64_t V, uint8_t* flags, uint32_t* out, uint32_t* nsel,
                                   void* temp, size_t temp_bytes, cudaStream_t st) {
    uint64_t blocks = (V + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (blocks < 1) blocks = 1;
    mask_flags_kernel<<<(unsigned)blocks, 256, 0, st>>>(mask, V, flags);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    return cub::DeviceSelect::Flagged(temp, temp_bytes, thrust::counting_iterator<uint32_t>(0), flags, out, nsel,
                                      (int64_t)V, st);
}

cudaError_t launch_mcmc(const McmcArgs& a, int num_sms, cudaStream_t st) {
    switch (a.nfibres) {
        case 1: return launch_mn<1>(a, num_sms, st);
        case 2: return launch_mn<2>(a, num_sms, st);
        case 3: return launch_mn<3>(a, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_samples_to_volume(const double* samples, const uint8_t* mask, uint64_t V, int N, int S,
                                     float* dyads, float* f, cudaStream_t st) {
    uint64_t blocks = ((uint64_t)N * S * V + 255) / 256;
    if (blocks > 148 * 32) blocks = 148 * 32;
    if (blocks < 1) blocks = 1;
    samples_to_volume_kernel<<<(unsigned)blocks, 256, 0, st>>>(samples, mask, V, N, S, dyads, f);
    return cudaGetLastError();
}

}  // namespace pt
