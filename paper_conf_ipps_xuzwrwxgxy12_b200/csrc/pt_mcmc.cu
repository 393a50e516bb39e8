// pt_mcmc.cu -- NEXT-4: Metropolis-Hastings sampling of the multiple partial volume model
// (Eq. 1; Sec. IV-A and Fig. 2) on sm_100a, binary64 (reading M4).
//
// The paper runs one thread per voxel.  Here one WARP owns a voxel and its lanes
// own the voxel's measurements (lane l holds i = l, l+32, ...): the per-measurement terms
// of Eq. 1 stay in registers for the whole chain (e^{-b d}, e^{-b d (r.v_j)^2}, r.v_j,
// the mixture A_i), so a proposal of S0, sigma or f_j costs no exponential at all, a
// proposal of an angle costs one per measurement and a proposal of d costs N+1; the sum of
// squared residuals is a warp reduction.  The NP draws of a loop do not depend on the state
// (counter-based Philox, M6), and omega'_k only depends on omega_k, which no other MH step
// of the loop changes: lane k computes draw k, the candidate and its transcendental
// by-products (ln sigma', sincos, ln|sin theta'|) for all NP steps of the loop in parallel
// at the loop's start; step k then only broadcasts them from lane k.
//
// Results follow contract C-MCMC of DESIGN.md §12 in the oracle's operation order; the
// oracle uses glibc's exp/log/sin/cos, this file CUDA's (both within an ulp or two), and
// the residual sum is a warp tree instead of a sequential loop, so samples agree to
// ~1e-13 relative rather than bit for bit (the parity bar of DESIGN.md §12).
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
constexpr int kMcmcThreads = 128;         // 4 voxels (warps) per CTA
#ifndef PT_MCMC_MIN_BLOCKS
#define PT_MCMC_MIN_BLOCKS 4  // CTAs per SM the register budget must allow (16 warps)
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

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return __shfl_sync(kFull, v, 0);  // one value for every lane (the butterfly's lanes may differ)
}

template <int N, int MPL>
__global__ void __launch_bounds__(kMcmcThreads, PT_MCMC_MIN_BLOCKS) mcmc_kernel(const __grid_constant__ McmcArgs a) {
    constexpr int NP = 3 + 3 * N;
    const uint32_t lane = threadIdx.x & 31u;
    const int n = a.nmeas;
    const double np1 = (double)(n + 1);

    // per-measurement data (registers): i = lane + 32 m
    bool valid[MPL];
    float yf[MPL], bf[MPL], rx[MPL], ry[MPL], rz[MPL];
#pragma unroll
    for (int m = 0; m < MPL; ++m) {
        const int i = (int)lane + 32 * m;
        valid[m] = i < n;
        bf[m] = valid[m] ? a.bvals[i] : 0.f;
        rx[m] = valid[m] ? a.bvecs[3 * i] : 0.f;
        ry[m] = valid[m] ? a.bvecs[3 * i + 1] : 0.f;
        rz[m] = valid[m] ? a.bvecs[3 * i + 2] : 0.f;
    }
    unsigned long long acc_tot = 0ull;

    for (;;) {
        uint32_t slot = 0;
        if (lane == 0) slot = atomicAdd(a.queue, 1u);
        slot = __shfl_sync(kFull, slot, 0);
        if (slot >= a.nvox) break;
        const uint32_t v = a.vox[slot];
        const uint64_t V = a.V;
#pragma unroll
        for (int m = 0; m < MPL; ++m) yf[m] = valid[m] ? a.dwi[(uint64_t)(lane + 32 * m) * V + v] : 0.f;

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
                if (bf[m] == 0.f) {
                    s0 += y;
                    c0 += 1;
                } else {
                    sd += y;
                    bsum += (double)bf[m];
                    cd += 1;
                }
            }
            s0 = warp_sum(s0);
            sd = warp_sum(sd);
            bsum = warp_sum(bsum);
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                c0 += __shfl_xor_sync(kFull, c0, o);
                cd += __shfl_xor_sync(kFull, cd, o);
                ymax = fmax(ymax, __shfl_xor_sync(kFull, ymax, o));
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
                    bool ok = valid[m] && bf[m] != 0.f;
#pragma unroll
                    for (int k = 0; k < j; ++k) {
                        const double dot = ((double)rx[m] * (double)px[k] + (double)ry[m] * (double)py[k]) +
                                           (double)rz[m] * (double)pz[k];
                        if (have[k]) ok = ok && fabs(dot) < 0.5;  // a missing pick constrains nothing
                    }
                    const int i = (int)lane + 32 * m;
                    if (ok && (yf[m] < by || (yf[m] == by && i < bi))) {
                        by = yf[m];
                        bi = i;
                    }
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    const float oy = __shfl_xor_sync(kFull, by, o);
                    const int oi = __shfl_xor_sync(kFull, bi, o);
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
        double e0[MPL], ej[N][MPL], dj[N][MPL], A[MPL];
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
            const double b = (double)bf[m];
            const double bd = b * w[1];
            e0[m] = exp(-bd);
            double acc = (1.0 - sumf) * e0[m];
#pragma unroll
            for (int j = 0; j < N; ++j) {
                const double vx = sth[j] * cph[j], vy = sth[j] * sph[j], vz = cth[j];
                dj[j][m] = madd((double)rz[m], vz, madd((double)ry[m], vy, (double)rx[m] * vx));
                ej[j][m] = exp(-(bd * (dj[j][m] * dj[j][m])));
                acc = madd(fj[j], ej[j][m], acc);
            }
            A[m] = acc;
            const double r = (double)yf[m] - w[0] * acc;
            sse = valid[m] ? madd(r, r, sse) : sse;
        }
        sse = warp_sum(sse);
        if (!a.init) {
            double sig = sqrt(sse / (double)n);
            if (!(sig >= 1e-3 * w[0])) sig = 1e-3 * w[0];
            w[2] = sig;
        }
        // uniform copies of the parameters the likelihood needs every step
        double S0 = w[0], dd = w[1], sig = w[2];
        double lsig = log(sig);
        double lp = -np1 * lsig - sse / (2.0 * sig * sig);
#pragma unroll
        for (int j = 0; j < N; ++j) lp = lp + lsin[j];

        // ------------------------------------------------ lane k owns parameter k: its value,
        // proposal width (M8), acceptance counters and, for angles, sin / cos (/ ln|sin|)
        double my_w = w[0];
#pragma unroll
        for (int k = 1; k < NP; ++k) my_w = lane == (uint32_t)k ? w[k] : my_w;
        double my_prop = 0.1;
        if (lane == 0u) my_prop = 0.01 * S0;
        else if (lane == 1u) my_prop = 0.1 * dd;
        else if (lane == 2u) my_prop = 0.1 * sig;
        else if (lane >= 3u && (lane - 3u) % 3u == 0u) my_prop = 0.05;
        double my_s = 0.0, my_c = 0.0;  // angle lanes: sin, cos of the current value
#pragma unroll
        for (int j = 0; j < N; ++j) {
            if (lane == (uint32_t)(4 + 3 * j)) {
                my_s = sth[j];
                my_c = cth[j];
            } else if (lane == (uint32_t)(5 + 3 * j)) {
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
            constexpr int B = 32 / NP;
            const uint32_t ph = t % (uint32_t)B;
            if (ph == 0u && lane < (uint32_t)(B * NP)) {
                const uint32_t tt = t + lane / (uint32_t)NP, kk = lane % (uint32_t)NP;
                const uint4 R = philox4x32_10(make_uint4(tt, v, kk, kTag), a.key0, a.key1);
                const double u1 = ((double)R.x + 0.5) * 0x1p-32;
                const double u2 = (double)R.y * 0x1p-32;
                const double u3 = ((double)R.z + 0.5) * 0x1p-32;
                bz = sqrt(-2.0 * log(u1)) * cos(kTwoPi * u2);
                blu = log(u3);
            }
            // lane k < NP: draw k of this loop, candidate omega'_k and its by-products
            const uint32_t src = ph * (uint32_t)NP + (lane < (uint32_t)NP ? lane : 0u);
            const double z = __shfl_sync(kFull, bz, src);
            const double clu = __shfl_sync(kFull, blu, src);
            double cz = 0.0, ca = 0.0, cb = 0.0, cc = 0.0;
            if (lane < (uint32_t)NP) {
                cz = my_w + my_prop * z;
                if (lane == 2u) {
                    ca = log(cz);
                } else if (lane >= 3u) {
                    const uint32_t r3 = (lane - 3u) % 3u;
                    if (r3 != 0u) {  // theta / phi: sin, cos (theta: and ln|sin|)
                        sincos(cz, &ca, &cb);
                        if (r3 == 1u) cc = log(fabs(ca));
                    }
                }
            }
            // Fig. 2: the MH step, repeated NumParameters times
#pragma unroll
            for (int k = 0; k < NP; ++k) {
                if (a.fixed & (1u << k)) continue;
                const double cand = __shfl_sync(kFull, cz, k);
                const double lu = __shfl_sync(kFull, clu, k);
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
                if (!ok) {
                    if (lane == (uint32_t)k) my_rej += 1u;
                    continue;
                }
                double xa = 0.0, xb = 0.0, xc = 0.0;  // the candidate's by-products (lane k)
                double nvx = 0.0, nvy = 0.0, nvz = 0.0;
                if (k == 2) {
                    xa = __shfl_sync(kFull, ca, k);
                } else if (r3 == 1 || r3 == 2) {
                    xa = __shfl_sync(kFull, ca, k);
                    xb = __shfl_sync(kFull, cb, k);
                    // the fibre's other angle, current value, from its owner lane
                    const int other = r3 == 1 ? k + 1 : k - 1;
                    const double os = __shfl_sync(kFull, my_s, other);
                    const double oc = __shfl_sync(kFull, my_c, other);
                    if (r3 == 1) {  // theta' with the current phi
                        xc = __shfl_sync(kFull, cc, k);
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
                double ne[MPL], nd[MPL], nA[MPL], nej[N][MPL];
                if (k == 2) {
                    nlp = -np1 * xa - sse / (2.0 * cand * cand);
#pragma unroll
                    for (int j = 0; j < N; ++j) nlp = nlp + lsin[j];
                } else {
#pragma unroll
                    for (int m = 0; m < MPL; ++m) {
                        double mu;
                        if (k == 0) {
                            mu = cand * A[m];
                        } else if (k == 1) {
                            const double bd = (double)bf[m] * cand;
                            ne[m] = exp(-bd);
                            double accm = (1.0 - sumf) * ne[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) {
                                nej[j][m] = exp(-(bd * (dj[j][m] * dj[j][m])));
                                accm = madd(fj[j], nej[j][m], accm);
                            }
                            nA[m] = accm;
                            mu = S0 * accm;
                        } else if (r3 == 0) {
                            double accm = (1.0 - nsumf) * e0[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) accm = madd(j == jf ? cand : fj[j], ej[j][m], accm);
                            nA[m] = accm;
                            mu = S0 * accm;
                        } else {
                            const double bd = (double)bf[m] * dd;
                            nd[m] = madd((double)rz[m], nvz, madd((double)ry[m], nvy, (double)rx[m] * nvx));
                            ne[m] = exp(-(bd * (nd[m] * nd[m])));
                            double accm = (1.0 - sumf) * e0[m];
#pragma unroll
                            for (int j = 0; j < N; ++j) accm = madd(fj[j], j == jf ? ne[m] : ej[j][m], accm);
                            nA[m] = accm;
                            mu = S0 * accm;
                        }
                        const double r = (double)yf[m] - mu;
                        nsse = valid[m] ? madd(r, r, nsse) : nsse;
                    }
                    nsse = warp_sum(nsse);
                    nlp = -np1 * lsig - nsse / (2.0 * sig * sig);
#pragma unroll
                    for (int j = 0; j < N; ++j) nlp = nlp + ((r3 == 1 && j == jf) ? xc : lsin[j]);
                }
                // accept with probability min(r, 1): ln u < lp' - lp
                const bool accept = lu < nlp - lp;
                if (lane == (uint32_t)k) {
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
                            A[m] = nA[m];
                        }
                    } else if (k == 2) {
                        sig = cand;
                        lsig = xa;
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
                            A[m] = nA[m];
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
                if (lane < (uint32_t)NP) a.samples[((uint64_t)lane * a.nsamples + s) * V + v] = my_w;
            }
        }
        if (a.accepted && lane < (uint32_t)NP) a.accepted[(uint64_t)lane * V + v] = my_tot;
        if (lane < (uint32_t)NP) acc_tot += my_tot;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc_tot += __shfl_xor_sync(kFull, acc_tot, o);
    if (lane == 0 && acc_tot) atomicAdd(a.stats + kMcmcStatAccepted, acc_tot);
}

template <int N, int MPL>
cudaError_t launch_m(const McmcArgs& a, int num_sms, cudaStream_t st) {
    auto k = mcmc_kernel<N, MPL>;
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kMcmcThreads, 0);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    const uint64_t need = ((uint64_t)a.nvox + kMcmcThreads / 32 - 1) / (kMcmcThreads / 32);
    const uint64_t full = (uint64_t)num_sms * (uint64_t)per_sm;
    const uint64_t grid = need < full ? need : full;
    if (grid == 0) return cudaSuccess;
    k<<<(unsigned)grid, kMcmcThreads, 0, st>>>(a);
    return cudaGetLastError();
}

template <int N>
cudaError_t launch_mn(const McmcArgs& a, int num_sms, cudaStream_t st) {
    switch ((a.nmeas + 31) / 32) {
        case 1: return launch_m<N, 1>(a, num_sms, st);
        case 2: return launch_m<N, 2>(a, num_sms, st);
        case 3: return launch_m<N, 3>(a, num_sms, st);
        case 4: return launch_m<N, 4>(a, num_sms, st);
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
