/*
 * oracle_mcmc.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * Plain single-threaded CPU reference of the paper's first GPU step (NEXT-4): Metropolis-
 * Hastings sampling of the multiple partial volume ("ball and stick") model, one voxel at
 * a time, one parameter at a time, exactly in the order of Sec. III-A and
 * Sec. IV-A / Fig. 2, with the readings M1-M9 of DESIGN.md §12.
 *
 * Double precision (binary64) throughout, libm exp/log/sin/cos/acos/atan2/sqrt, no FMA
 * contraction (-ffp-contract=off).  Nothing here is blocked, cached or reordered: every
 * proposal recomputes the whole log-posterior from the data.
 */
#include "oracle.h"

#include <math.h>
#include <stddef.h>
#include <string.h>

#define MCMC_TAG 0x4D434D43u  /* "MCMC": Philox counter word 3 of the sampler's draws (M6) */
#define TWO_PI 6.283185307179586

/* Eq. 1: mu_i = S0 [ (1 - sum_j f_j) exp(-b_i d) + sum_j f_j exp(-b_i d (r_i.v_j)^2) ],
 * v_j = (sin th cos ph, sin th sin ph, cos th).  omega = (S0, d, sigma, f_1, th_1, ph_1, ...). */
void oracle_mcmc_signal(int nfibres, const double* w, int n, const float* bvals, const float* bvecs,
                        double* mu) {
    int i, j;
    double sumf = 0.0;
    for (j = 0; j < nfibres; ++j) sumf = sumf + w[3 + 3 * j];
    for (i = 0; i < n; ++i) {
        const double b = (double)bvals[i];
        const double rx = (double)bvecs[3 * i], ry = (double)bvecs[3 * i + 1], rz = (double)bvecs[3 * i + 2];
        const double bd = b * w[1];
        double acc = (1.0 - sumf) * exp(-bd);
        for (j = 0; j < nfibres; ++j) {
            const double th = w[4 + 3 * j], ph = w[5 + 3 * j];
            const double vx = sin(th) * cos(ph), vy = sin(th) * sin(ph), vz = cos(th);
            const double dot = (rx * vx + ry * vy) + rz * vz;
            acc = acc + w[3 + 3 * j] * exp(-(bd * (dot * dot)));
        }
        mu[i] = w[0] * acc;
    }
}

/* M3: support of the priors: S0 > 0, d > 0, sigma > 0, f_j >= 0, sum f_j <= 1. */
static int in_support(int nfibres, const double* w) {
    int j;
    double sumf = 0.0;
    if (!(w[0] > 0.0) || !(w[1] > 0.0) || !(w[2] > 0.0)) return 0;
    for (j = 0; j < nfibres; ++j) {
        if (!(w[3 + 3 * j] >= 0.0)) return 0;
        sumf = sumf + w[3 + 3 * j];
    }
    return sumf <= 1.0;
}

/* M2/M3: log P(omega | Y) up to a constant: Gaussian likelihood of Eq. 1 with noise standard
 * deviation sigma (the ninth parameter), Jeffreys prior 1/sigma, uniform S0, d, f,
 * orientation uniform on the sphere (density |sin th| in (th, ph)). */
static double log_post(int nfibres, const double* w, int n, const double* y, const float* bvals,
                       const float* bvecs, double* mu) {
    int i, j;
    double sse = 0.0, lp;
    oracle_mcmc_signal(nfibres, w, n, bvals, bvecs, mu);
    for (i = 0; i < n; ++i) {
        const double r = y[i] - mu[i];
        sse = sse + r * r;
    }
    lp = -(double)(n + 1) * log(w[2]) - sse / (2.0 * w[2] * w[2]);
    for (j = 0; j < nfibres; ++j) lp = lp + log(fabs(sin(w[4 + 3 * j])));
    return lp;
}

/* M6: the three uniforms of one MH step (two for the Box-Muller Gaussian of the
 * proposal, one for the acceptance test), from one Philox4x32-10 block with counter
 * {loop, voxel, k, "MCMC"}.  z = sqrt(-2 ln u1) cos(2 pi u2) (Box-Muller [36]). */
void oracle_mcmc_draw(uint64_t seed, uint32_t loop, uint32_t voxel, uint32_t k, double* z, double* logu) {
    const uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    const uint32_t ctr[4] = {loop, voxel, k, MCMC_TAG};
    uint32_t w[4];
    double u1, u2, u3;
    oracle_philox4x32_10(ctr, key, w);
    u1 = ((double)w[0] + 0.5) * 0x1p-32;  /* (0, 1): never 0 */
    u2 = (double)w[1] * 0x1p-32;           /* [0, 1) */
    u3 = ((double)w[2] + 0.5) * 0x1p-32;  /* (0, 1) */
    *z = sqrt(-2.0 * log(u1)) * cos(TWO_PI * u2);
    *logu = log(u3);
}

/* M7: automatic initial state of a voxel (the paper does not say how the chain starts). */
static void initial_state(int nfibres, int n, const double* y, const float* bvals, const float* bvecs,
                          double* w, double* mu) {
    int i, j, cnt0 = 0, cntd = 0;
    double s0 = 0.0, ymax = -HUGE_VAL, sd = 0.0, bsum = 0.0, d, sse = 0.0, sig;
    int best[3] = {-1, -1, -1};
    for (i = 0; i < n; ++i) {
        if (y[i] > ymax) ymax = y[i];
        if (bvals[i] == 0.0f) {
            s0 = s0 + y[i];
            cnt0 += 1;
        } else {
            sd = sd + y[i];
            bsum = bsum + (double)bvals[i];
            cntd += 1;
        }
    }
    /* S0 = mean of the b = 0 measurements (else the largest measurement) */
    s0 = cnt0 ? s0 / (double)cnt0 : ymax;
    if (!(s0 > 0.0)) s0 = 1.0;
    /* d from the mean attenuation of the diffusion-weighted measurements */
    d = 0.0;
    if (cntd) d = -log((sd / (double)cntd) / s0) / (bsum / (double)cntd);
    if (!(d > 0.0) || !isfinite(d)) d = cntd ? 1.0 / (bsum / (double)cntd) : 1.0;
    /* fibre j: the diffusion-weighted direction of the smallest signal (strongest
     * attenuation) among those with |r . v_k| < 0.5 for every earlier fibre k */
    for (j = 0; j < nfibres; ++j) {
        double ybest = HUGE_VAL;
        for (i = 0; i < n; ++i) {
            int k, ok = bvals[i] != 0.0f;
            for (k = 0; k < j && ok; ++k) {
                const int m = best[k];
                double dot;
                if (m < 0) continue;              /* no earlier pick: no constraint (M7) */
                dot = ((double)bvecs[3 * i] * (double)bvecs[3 * m] +
                                    (double)bvecs[3 * i + 1] * (double)bvecs[3 * m + 1]) +
                                   (double)bvecs[3 * i + 2] * (double)bvecs[3 * m + 2];
                if (!(fabs(dot) < 0.5)) ok = 0;
            }
            if (ok && y[i] < ybest) {
                ybest = y[i];
                best[j] = i;
            }
        }
    }
    w[0] = s0;
    w[1] = d;
    for (j = 0; j < nfibres; ++j) {
        w[3 + 3 * j] = j == 0 ? 0.3 : 0.1;
        if (best[j] >= 0) {
            const double rz = (double)bvecs[3 * best[j] + 2];
            w[4 + 3 * j] = acos(rz < -1.0 ? -1.0 : (rz > 1.0 ? 1.0 : rz));
            w[5 + 3 * j] = atan2((double)bvecs[3 * best[j] + 1], (double)bvecs[3 * best[j]]);
        } else if (j == 0) {
            w[4] = 1.0;
            w[5] = 0.0;
        } else {            /* no direction left: turn fibre 0 by 90 degrees */
            w[4 + 3 * j] = w[4] + (j == 1 ? 1.5707963267948966 : 0.0);
            w[5 + 3 * j] = w[5] + (j == 2 ? 1.5707963267948966 : 0.0);
        }
    }
    /* sigma = RMS residual of the initial model, at least 1e-3 S0 */
    w[2] = 1.0;
    oracle_mcmc_signal(nfibres, w, n, bvals, bvecs, mu);
    for (i = 0; i < n; ++i) sse = sse + (y[i] - mu[i]) * (y[i] - mu[i]);
    sig = sqrt(sse / (double)n);
    if (!(sig >= 1e-3 * s0)) sig = 1e-3 * s0;
    w[2] = sig;
}

int oracle_mcmc(const oracle_dwi* dw, const oracle_mcmc_params* p, const double* init,
                int64_t v_begin, int64_t v_end, double* samples, uint32_t* accepted) {
    const int N = p->nfibres;
    const int NP = 3 + 3 * N;
    const int n = dw->nmeas;
    const int64_t V = (int64_t)dw->nx * dw->ny * dw->nz;
    const int64_t loops = (int64_t)p->burnin + (int64_t)p->nsamples * p->interval;
    double y[ORACLE_MCMC_MAX_MEAS], mu[ORACLE_MCMC_MAX_MEAS];
    int64_t v;

    if (N < 1 || N > 3 || n < 1 || n > ORACLE_MCMC_MAX_MEAS) return -1;
    if (p->burnin < 0 || p->nsamples < 1 || p->interval < 1 || p->adapt_every < 1) return -1;
    if (loops > 0xFFFFFFFFll) return -1;
    if (v_begin < 0 || v_end > V || v_end < v_begin) return -2;

    for (v = v_begin; v < v_end; ++v) {
        double w[12], wn[12], prop[12], lp;
        uint32_t acc[12], rej[12], acc_tot[12];
        int64_t t;
        int i, k;
        if (dw->mask[v] == 0) continue;
        for (i = 0; i < n; ++i) y[i] = (double)dw->dwi[(int64_t)i * V + v];
        if (init) {
            for (k = 0; k < NP; ++k) w[k] = init[(int64_t)k * V + v];
        } else {
            initial_state(N, n, y, dw->bvals, dw->bvecs, w, mu);
        }
        /* M8: initial proposal standard deviations */
        prop[0] = 0.01 * w[0];
        prop[1] = 0.1 * w[1];
        prop[2] = 0.1 * w[2];
        for (k = 0; k < N; ++k) {
            prop[3 + 3 * k] = 0.05;
            prop[4 + 3 * k] = 0.1;
            prop[5 + 3 * k] = 0.1;
        }
        memset(acc, 0, sizeof acc);
        memset(rej, 0, sizeof rej);
        memset(acc_tot, 0, sizeof acc_tot);
        lp = log_post(N, w, n, y, dw->bvals, dw->bvecs, mu);

        for (t = 0; t < loops; ++t) {
            /* Fig. 2: in each loop the MH step is repeated NumParameters times */
            for (k = 0; k < NP; ++k) {
                double z, logu, lpn;
                if (p->fixed & (1u << k)) continue;
                oracle_mcmc_draw(p->rng_seed, (uint32_t)t, (uint32_t)v, (uint32_t)k, &z, &logu);
                /* propose omega' from N(omega_k, prop_k^2) */
                memcpy(wn, w, sizeof(double) * (size_t)NP);
                wn[k] = w[k] + prop[k] * z;
                if (!in_support(N, wn)) {
                    rej[k] += 1;
                    continue;
                }
                /* accept with probability min(r, 1), r = P(omega'|Y) / P(omega|Y) */
                lpn = log_post(N, wn, n, y, dw->bvals, dw->bvecs, mu);
                if (logu < lpn - lp) {
                    w[k] = wn[k];
                    lp = lpn;
                    acc[k] += 1;
                    acc_tot[k] += 1;
                } else {
                    rej[k] += 1;
                }
            }
            /* Fig. 2: every K loops the acceptance rates update the proposals (keep
             * the rate between 25% and 50%; M8: the fixed point is 37.5%) */
            if ((t + 1) % p->adapt_every == 0) {
                for (k = 0; k < NP; ++k) {
                    prop[k] = prop[k] * sqrt((5.0 * (double)(acc[k] + 1u)) / (3.0 * (double)(rej[k] + 1u)));
                    acc[k] = 0;
                    rej[k] = 0;
                }
            }
            /* samples after the burn-in, every L loops */
            if (t >= p->burnin && (t - p->burnin + 1) % p->interval == 0) {
                const int64_t s = (t - p->burnin + 1) / p->interval - 1;
                for (k = 0; k < NP; ++k) samples[((int64_t)k * p->nsamples + s) * V + v] = w[k];
            }
        }
        if (accepted)
            for (k = 0; k < NP; ++k) accepted[(int64_t)k * V + v] = acc_tot[k];
    }
    return 0;
}
