/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * A plain transcription of the per-particle streamlining loop: Algorithm 1's inner loop
 * (Interpolation(); StepToNextPoint(); stop test), with the probabilistic
 * streamlining semantics of Sec. III-B and the readings R1-R20 of DESIGN.md.
 * No blocking, no batching, no reordering: one particle at a time, one step at a time.
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math (no FMA contraction, no
 * FTZ/DAZ, SSE float arithmetic with FLT_EVAL_METHOD == 0): every float operation below
 * is a single IEEE-754 binary32 operation rounded to nearest-even (R15).
 */
#include "oracle.h"

#include <float.h>
#include <math.h>
#include <stddef.h>
#include <string.h>

#if !defined(FLT_EVAL_METHOD) || FLT_EVAL_METHOD != 0
#error "oracle needs FLT_EVAL_METHOD == 0 (binary32 evaluation)"
#endif

/* ------------------------------------------------------------------ R16: Philox4x32-10
 * Salmon, Moraes, Dror, Shaw, "Parallel random numbers: as easy as 1, 2, 3" (SC'11),
 * the Random123 reference round:  (c0,c1,c2,c3) ->
 *   (hi(M1*c2) ^ c1 ^ k0,  lo(M1*c2),  hi(M0*c0) ^ c3 ^ k1,  lo(M0*c0)),
 * ten rounds, the key bumped by the Weyl constants between rounds.  Replaces the
 * paper's combined Tausworthe generator for the tracking draws. */
void oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
    uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
    uint32_t k0 = key[0], k1 = key[1];
    int r;
    for (r = 0; r < 10; ++r) {
        uint64_t p0, p1;
        uint32_t n0, n1, n2, n3;
        if (r > 0) {
            k0 = k0 + 0x9E3779B9u;
            k1 = k1 + 0xBB67AE85u;
        }
        p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
        p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
        n0 = (uint32_t)(p1 >> 32) ^ c1 ^ k0;
        n1 = (uint32_t)p1;
        n2 = (uint32_t)(p0 >> 32) ^ c3 ^ k1;
        n3 = (uint32_t)p0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* R16: s = floor(w * S / 2^32) -- integer only, so both sides agree exactly. */
uint32_t oracle_sample_index(uint32_t w, uint32_t nsamples) {
    return (uint32_t)(((uint64_t)w * (uint64_t)nsamples) >> 32);
}

/* ------------------------------------------------------------------ R15: binary16 decode
 * IEEE 754-2008 binary16: 1 sign, 5 exponent (bias 15), 10 fraction bits.  Every half
 * value is exactly representable in binary32, so the decode is exact. */
float oracle_half_to_float(uint16_t h) {
    uint32_t sign = (uint32_t)(h >> 15) & 1u;
    uint32_t e = (uint32_t)(h >> 10) & 0x1Fu;
    uint32_t m = (uint32_t)h & 0x3FFu;
    float v;
    if (e == 0u) {
        v = ldexpf((float)m, -24);                    /* zero / subnormal: m * 2^-24 */
    } else if (e == 31u) {
        v = (m != 0u) ? NAN : INFINITY;
    } else {
        v = ldexpf((float)(m | 0x400u), (int)e - 25); /* (1024 + m) * 2^(e-15-10) */
    }
    return sign ? -v : v;
}

void oracle_half_to_float_array(const uint16_t* h, float* out, int64_t n) {
    int64_t i;
    for (i = 0; i < n; ++i) out[i] = oracle_half_to_float(h[i]);
}

/* ------------------------------------------------------------------ R10: voxel lookup
 * Positions are kept in centred coordinates q = x - c, c = floor(N/2).  The voxel index
 * along an axis is c + trunc(q) - signbit(q): voxel i covers [i-c, i-c+1) for i >= c and
 * (i-c, i-c+1] for i < c; +0 belongs to voxel c, -0 to voxel c-1. */
int64_t oracle_axis_index(float q, int32_t n_axis) {
    int64_t c = (int64_t)(n_axis / 2);
    if (!(fabsf(q) < 1.0e9f)) return -1;              /* far outside (or NaN) */
    return c + (int64_t)truncf(q) - (signbit(q) ? 1 : 0);
}

/* voxel lookup + bounds + mask ("Meet the Stop Criteria"; R11): returns the
 * linear voxel index [Z][Y][X], or -1 if outside the volume or outside the mask. */
static int64_t lookup(const oracle_volume* v, const float q[3]) {
    int64_t ix = oracle_axis_index(q[0], v->nx);
    int64_t iy = oracle_axis_index(q[1], v->ny);
    int64_t iz = oracle_axis_index(q[2], v->nz);
    int64_t idx;
    if (ix < 0 || ix >= v->nx || iy < 0 || iy >= v->ny || iz < 0 || iz >= v->nz) return -1;
    idx = (iz * v->ny + iy) * v->nx + ix;
    if (v->mask[idx] == 0) return -1;
    return idx;
}

/* "Interpolation()" of Alg. 1, nearest voxel (R2): fetch fibre j's direction
 * and fraction of sample s at voxel vox from the sample volumes. */
static void fetch(const oracle_volume* v, int64_t vox, uint32_t s, int j, float dir[3], float* fj) {
    int64_t V = (int64_t)v->nx * v->ny * v->nz;
    int64_t e = ((int64_t)j * v->nsamples + s) * V + vox;
    int a;
    if (v->is_half) {
        const uint16_t* d = (const uint16_t*)v->dyads;
        const uint16_t* f = (const uint16_t*)v->f;
        for (a = 0; a < 3; ++a) dir[a] = oracle_half_to_float(d[e * 3 + a]);
        *fj = oracle_half_to_float(f[e]);
    } else {
        const float* d = (const float*)v->dyads;
        const float* f = (const float*)v->f;
        for (a = 0; a < 3; ++a) dir[a] = d[e * 3 + a];
        *fj = f[e];
    }
}

static int valid_params(const oracle_volume* v, const oracle_params* p) {
    if (v->nx <= 0 || v->ny <= 0 || v->nz <= 0) return 0;
    if (v->nsamples < 1 || v->nfibres < 1 || v->nfibres > 3) return 0;
    if (!(p->step > 0.0f) || !isfinite(p->step)) return 0;
    if (!(fabsf(p->curv_thr) <= 1.0f)) return 0;
    if (isnan(p->fib_thr)) return 0;
    if (p->max_steps < 1 || p->max_steps > 65535) return 0;
    if (p->particles_per_seed < 1) return 0;
    if (p->sample_mode != 0 && p->sample_mode != 1) return 0;
    return 1;
}

int oracle_track(const oracle_volume* vol, const oracle_params* prm,
                 const float* seeds_xyz, const uint64_t* seed_ids, int64_t nseeds,
                 int64_t j_begin, int64_t j_end,
                 uint64_t* map, int32_t* nsteps, uint8_t* reason, float* end_xyz,
                 float* paths, int32_t path_stride,
                 const uint8_t* labels, int32_t ntargets, uint64_t* conn) {
    const int F = vol->nfibres;
    const uint32_t S = (uint32_t)vol->nsamples;
    const uint64_t P = (uint64_t)prm->particles_per_seed;
    const uint32_t key[2] = {(uint32_t)prm->rng_seed, (uint32_t)(prm->rng_seed >> 32)};
    const float c[3] = {(float)(vol->nx / 2), (float)(vol->ny / 2), (float)(vol->nz / 2)};
    const int64_t npp = j_end - j_begin;
    int64_t si, jj;

    if (!valid_params(vol, prm)) return -1;
    if (nseeds < 0 || j_begin < 0 || j_end < j_begin || (uint64_t)j_end > P) return -2;
    if (paths && path_stride < 1) return -3;
    if (conn && (!labels || ntargets < 1 || ntargets > 64)) return -5;

    for (si = 0; si < nseeds; ++si) {
        const uint64_t sid = seed_ids ? seed_ids[si] : (uint64_t)si;
        if (sid > (UINT64_MAX - (P - 1)) / P) return -4;       /* pid overflow */
        for (jj = j_begin; jj < j_end; ++jj) {
            const uint64_t pid = sid * P + (uint64_t)jj;         /* particle id */
            const int64_t out = si * npp + (jj - j_begin);
            const uint32_t plo = (uint32_t)pid, phi = (uint32_t)(pid >> 32);
            float q[3], p[3] = {0.0f, 0.0f, 0.0f};
            unsigned char entered[64];   /* NEXT-2: targets this streamline passed through */
            int64_t vox;
            int32_t n = 0;
            int why;
            int a;

            memset(entered, 0, sizeof entered);
            /* GetStartPoint(): centred coordinates q = x - c (R10). */
            for (a = 0; a < 3; ++a) q[a] = seeds_xyz[si * 3 + a] - c[a];
            if (paths) {
                int32_t k;
                for (k = 0; k < path_stride * 3; ++k) paths[out * path_stride * 3 + k] = NAN;
                for (a = 0; a < 3; ++a) paths[out * path_stride * 3 + a] = q[a] + c[a];
            }
            vox = lookup(vol, q);
            if (vox < 0) {
                why = ORACLE_END_MASK;                           /* R12: seed outside */
            } else {
                for (;;) {
                    uint32_t blk_ctr[4], w[4];
                    uint32_t s;
                    float v[3][3], fv[3];
                    float d[3], qn[3];
                    int jstar, j;
                    float sgn;
                    int64_t vn;

                    /* maximum number of steps (R14) -- checked first */
                    if (n == prm->max_steps) { why = ORACLE_END_MAXLEN; break; }

                    /* R1/R16: a fresh random sample index every step.  Block b = n/3 of
                     * the particle's stream: ctr = {b, pid_lo, pid_hi, 0}; word n%3. */
                    blk_ctr[0] = (uint32_t)(n / 3); blk_ctr[1] = plo; blk_ctr[2] = phi; blk_ctr[3] = 0u;
                    oracle_philox4x32_10(blk_ctr, key, w);
                    if (prm->sample_mode == 1)
                        s = (uint32_t)((uint64_t)jj % S);   /* NEXT-1: one sample volume per
                                                               streamline */
                    else
                        s = oracle_sample_index(w[n % 3], S);

                    /* Interpolation() (R2): the sample's fibres at this voxel */
                    for (j = 0; j < F; ++j) fetch(vol, vox, s, j, v[j], &fv[j]);

                    if (n == 0) {
                        /* R5, R6: first step follows fibre 0 with a random sign: the top
                         * bit of word 3 of block 0 (w holds block 0 here). */
                        jstar = 0;
                        sgn = (w[3] >> 31) ? -1.0f : 1.0f;
                    } else {
                        /* choose the fibre closest to the previous direction
                         * (R7 eligibility f_j > fib_thr, R8 strict >, lowest j on ties). */
                        float cj[3];
                        float best = -1.0f;
                        jstar = -1;
                        for (j = 0; j < F; ++j) {
                            cj[j] = (v[j][0] * p[0] + v[j][1] * p[1]) + v[j][2] * p[2];
                            if (fv[j] > prm->fib_thr && fabsf(cj[j]) > best) {
                                best = fabsf(cj[j]);
                                jstar = j;
                            }
                        }
                        if (jstar < 0) jstar = 0;                 /* R7: none eligible */
                        /* maximum angle, measured by the dot product (R4) */
                        if (!(fabsf(cj[jstar]) > prm->curv_thr)) { why = ORACLE_END_CURV; break; }
                        /* keep the streamline's orientation (R9) */
                        sgn = (cj[jstar] > 0.0f) ? 1.0f : -1.0f;
                    }

                    /* StepToNextPoint(): q' = q + h * d, d = sgn * v */
                    for (a = 0; a < 3; ++a) {
                        d[a] = sgn * v[jstar][a];
                        qn[a] = q[a] + prm->step * d[a];
                    }

                    /* stop test at the candidate position (R11): the failing
                     * step is not committed */
                    vn = lookup(vol, qn);
                    if (vn < 0) { why = ORACLE_END_MASK; break; }

                    /* commit; count one visit of the new voxel (R13) */
                    for (a = 0; a < 3; ++a) { q[a] = qn[a]; p[a] = d[a]; }
                    vox = vn;
                    n = n + 1;
                    if (map) map[vox] += 1u;
                    if (conn && labels[vox] != 0 && labels[vox] <= ntargets)
                        entered[labels[vox] - 1] = 1;     /* R21: committed steps only */
                    if (paths && n < path_stride) {
                        for (a = 0; a < 3; ++a) paths[(out * path_stride + n) * 3 + a] = q[a] + c[a];
                    }
                }
            }
            /* SetEndPoint() */
            if (nsteps) nsteps[out] = n;
            if (reason) reason[out] = (uint8_t)why;
            if (end_xyz) for (a = 0; a < 3; ++a) end_xyz[out * 3 + a] = q[a] + c[a];
            /* count the streamlines passing through each target, once each */
            if (conn) {
                int t;
                for (t = 0; t < ntargets; ++t)
                    if (entered[t]) conn[si * ntargets + t] += 1u;
            }
        }
    }
    return 0;
}
