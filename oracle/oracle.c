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
#include <stdlib.h>
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

/* NEXT-3, R23: probabilistic interpolation of the sampled voxel ("Interpolation()",
 * P:L175, in FSL's probabilistic form).  Along each axis the position q lies between the
 * centres of two voxels (centre of voxel c+k is q = k + 0.5); the upper one is taken with
 * probability equal to its linear-interpolation weight:
 *   t = q - 0.5 (one fp32 RNE subtraction),  m = floor(t),  fr = t - m,
 *   r = (w >> 8) * 2^-24 (exact uniform in [0,1)),  index = c + m + (r < fr ? 1 : 0).
 * Returns the linear voxel index, or -1 if that voxel is outside the volume or the mask
 * (the caller then falls back to the nearest voxel). */
static int64_t interp_voxel(const oracle_volume* v, const float q[3], const uint32_t w[4]) {
    const int32_t N[3] = {v->nx, v->ny, v->nz};
    int64_t idx[3], lin;
    int a;
    for (a = 0; a < 3; ++a) {
        float t = q[a] - 0.5f;
        float m = floorf(t);
        float fr = t - m;
        float r = (float)(w[a] >> 8) * 0x1p-24f;
        idx[a] = (int64_t)(N[a] / 2) + (int64_t)m + (r < fr ? 1 : 0);
        if (idx[a] < 0 || idx[a] >= N[a]) return -1;
    }
    lin = (idx[2] * v->ny + idx[1]) * v->nx + idx[0];
    if (v->mask[lin] == 0) return -1;
    return lin;
}

/* NEXT-3, R24: fibre of the very first step.  Eligible fibres E = {j : f_j > fib_thr} in
 * index order.  mode 0: fibre 0 (R5).  mode 1: E[floor(w |E| / 2^32)].  mode 2: the first
 * j in E with r < f_E0 + ... + f_j (fp32 sums left to right), r = u * sum_E f (fp32),
 * u = (w >> 8) * 2^-24; the last of E if rounding leaves none.  E empty: fibre 0. */
static int initial_fibre(int mode, int F, const float fv[3], float fib_thr, uint32_t w) {
    int elig[3], ne = 0, j, k;
    float tot = 0.0f, r, cum = 0.0f;
    for (j = 0; j < F; ++j)
        if (fv[j] > fib_thr) elig[ne++] = j;
    if (mode == 0 || ne == 0) return 0;
    if (mode == 1) return elig[(uint32_t)(((uint64_t)w * (uint64_t)ne) >> 32)];
    for (k = 0; k < ne; ++k) tot = tot + fv[elig[k]];
    r = ((float)(w >> 8) * 0x1p-24f) * tot;
    for (k = 0; k < ne; ++k) {
        cum = cum + fv[elig[k]];
        if (r < cum) return elig[k];
    }
    return elig[ne - 1];
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
    if (p->bidir != 0 && p->bidir != 1) return 0;
    if (p->interp != 0 && p->interp != 1) return 0;
    if (p->init_fibre < 0 || p->init_fibre > 2) return 0;
    return 1;
}

/* Everything one half-streamline needs besides the volume and parameters. */
typedef struct {
    uint64_t pid;            /* particle id = seed_id * P + j (RNG counter, R16)        */
    int64_t j;               /* particle index within its seed (paper mode, NEXT-1)     */
    int half;                /* 0, or 1 = the reverse half of a bidirectional streamline */
    float seed[3];           /* seed, corner coordinates                                 */
    float d0[3];             /* in/out: half 0's first step direction (R22)              */
    int have_d0;             /* in/out                                                   */
    unsigned char* entered;  /* [64] targets entered (NEXT-2) or NULL                    */
    uint64_t* map;
    const uint8_t* labels;
    int32_t ntargets;
    float* path;             /* [path_stride][3] or NULL                                 */
    int32_t path_stride;
    int64_t* entered_vox;    /* R25: voxel of every committed step of the streamline, or NULL */
    int64_t nentered;
} half_io;

/* One (half-)streamline: Algorithm 1's inner loop.  Returns n; *why and the
 * end position (centred) are written. */
static int32_t track_half(const oracle_volume* vol, const oracle_params* prm, half_io* io,
                          int* why_out, float qend[3]) {
    const int F = vol->nfibres;
    const uint32_t S = (uint32_t)vol->nsamples;
    const uint32_t key[2] = {(uint32_t)prm->rng_seed, (uint32_t)(prm->rng_seed >> 32)};
    const float c[3] = {(float)(vol->nx / 2), (float)(vol->ny / 2), (float)(vol->nz / 2)};
    const uint32_t plo = (uint32_t)io->pid, phi = (uint32_t)(io->pid >> 32);
    const uint32_t h = (uint32_t)io->half;
    float q[3], p[3] = {0.0f, 0.0f, 0.0f};
    int64_t vox;
    int32_t n = 0;
    int why;
    int a;

    /* GetStartPoint(): centred coordinates q = x - c (R10). */
    for (a = 0; a < 3; ++a) q[a] = io->seed[a] - c[a];
    if (io->path) {
        int32_t k;
        for (k = 0; k < io->path_stride * 3; ++k) io->path[k] = NAN;
        for (a = 0; a < 3; ++a) io->path[a] = q[a] + c[a];
    }
    /* R22: the reverse half starts with previous direction -d0 */
    if (h == 1)
        for (a = 0; a < 3; ++a) p[a] = -io->d0[a];
    vox = lookup(vol, q);
    if (vox < 0 || (h == 1 && !io->have_d0)) {
        why = ORACLE_END_MASK;                               /* R12: seed outside */
    } else {
        for (;;) {
            uint32_t blk_ctr[4], w[4], wi[4] = {0u, 0u, 0u, 0u};
            uint32_t s;
            float v[3][3], fv[3];
            float d[3], qn[3];
            int jstar, j;
            float sgn;
            int64_t vn, vs;
            const int first = (n == 0 && h == 0);

            /* maximum number of steps (R14) -- checked first */
            if (n == prm->max_steps) { why = ORACLE_END_MAXLEN; break; }

            /* R1/R16: a fresh random sample index every step.  Block b = n/3 of the
             * half's stream: ctr = {b, pid_lo, pid_hi, half}; word n%3. */
            blk_ctr[0] = (uint32_t)(n / 3); blk_ctr[1] = plo; blk_ctr[2] = phi; blk_ctr[3] = h;
            oracle_philox4x32_10(blk_ctr, key, w);
            if (prm->sample_mode == 1)
                s = (uint32_t)((uint64_t)io->j % S);    /* NEXT-1: one sample volume per
                                                           streamline */
            else
                s = oracle_sample_index(w[n % 3], S);

            /* R23/R24 draws: stream 2 + half, block n (words 0-2: interpolation of
             * step n; word 3 of half 0's block 0: the first fibre) */
            if (prm->interp || (first && prm->init_fibre != 0)) {
                uint32_t ic[4];
                ic[0] = (uint32_t)n; ic[1] = plo; ic[2] = phi; ic[3] = 2u + h;
                oracle_philox4x32_10(ic, key, wi);
            }

            /* Interpolation(): nearest voxel (R2), or the probabilistic
             * neighbour (R23) with the nearest voxel as fallback */
            vs = vox;
            if (prm->interp) {
                int64_t u = interp_voxel(vol, q, wi);
                if (u >= 0) vs = u;
            }
            for (j = 0; j < F; ++j) fetch(vol, vs, s, j, v[j], &fv[j]);

            if (first) {
                /* R5/R24: the first fibre; R6: random sign, the top bit of word 3 of
                 * block 0 (w holds block 0 here). */
                jstar = initial_fibre(prm->init_fibre, F, fv, prm->fib_thr, wi[3]);
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
            if (first) {                                  /* R22: remember d0 */
                for (a = 0; a < 3; ++a) io->d0[a] = d[a];
                io->have_d0 = 1;
            }

            /* stop test at the candidate position (R11): the failing
             * step is not committed */
            vn = lookup(vol, qn);
            if (vn < 0) { why = ORACLE_END_MASK; break; }

            /* commit; count one visit of the new voxel (R13) */
            for (a = 0; a < 3; ++a) { q[a] = qn[a]; p[a] = d[a]; }
            vox = vn;
            n = n + 1;
            if (io->map) io->map[vox] += 1u;
            if (io->entered && io->labels[vox] != 0 && io->labels[vox] <= io->ntargets)
                io->entered[io->labels[vox] - 1] = 1;     /* R21: committed steps only */
            if (io->entered_vox) io->entered_vox[io->nentered++] = vox;  /* R25 */
            if (io->path && n < io->path_stride)
                for (a = 0; a < 3; ++a) io->path[n * 3 + a] = q[a] + c[a];
        }
    }
    *why_out = why;
    for (a = 0; a < 3; ++a) qend[a] = q[a];
    return n;
}

static int cmp_i64(const void* a, const void* b) {
    const int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
    return (x > y) - (x < y);
}

int oracle_track(const oracle_volume* vol, const oracle_params* prm,
                 const float* seeds_xyz, const uint64_t* seed_ids, int64_t nseeds,
                 int64_t j_begin, int64_t j_end,
                 uint64_t* map, int32_t* nsteps, uint8_t* reason, float* end_xyz,
                 float* paths, int32_t path_stride,
                 const uint8_t* labels, int32_t ntargets, uint64_t* conn, uint64_t* umap) {
    const uint64_t P = (uint64_t)prm->particles_per_seed;
    const float c[3] = {(float)(vol->nx / 2), (float)(vol->ny / 2), (float)(vol->nz / 2)};
    const int64_t npp = j_end - j_begin;
    const int halves = prm->bidir ? 2 : 1;
    int64_t si, jj;

    if (!valid_params(vol, prm)) return -1;
    if (nseeds < 0 || j_begin < 0 || j_end < j_begin || (uint64_t)j_end > P) return -2;
    if (paths && path_stride < 1) return -3;
    if (conn && (!labels || ntargets < 1 || ntargets > 64)) return -5;
    int64_t* entered_vox = NULL;  /* R25: committed-step voxels of one streamline */
    if (umap) {
        entered_vox = (int64_t*)malloc(sizeof(int64_t) * (size_t)halves * (size_t)prm->max_steps + 8);
        if (!entered_vox) return -6;
    }

    for (si = 0; si < nseeds; ++si) {
        const uint64_t sid = seed_ids ? seed_ids[si] : (uint64_t)si;
        if (sid > (UINT64_MAX - (P - 1)) / P) {                  /* pid overflow */
            free(entered_vox);
            return -4;
        }
        for (jj = j_begin; jj < j_end; ++jj) {
            const int64_t out = si * npp + (jj - j_begin);
            unsigned char entered[64];   /* NEXT-2: targets this streamline passed through */
            half_io io;
            int h, a;

            memset(entered, 0, sizeof entered);
            memset(&io, 0, sizeof io);
            io.pid = sid * P + (uint64_t)jj;                     /* particle id */
            io.j = jj;
            for (a = 0; a < 3; ++a) io.seed[a] = seeds_xyz[si * 3 + a];
            io.entered = conn ? entered : NULL;
            io.map = map;
            io.labels = labels;
            io.ntargets = ntargets;
            io.path_stride = path_stride;
            io.entered_vox = entered_vox;
            io.nentered = 0;
            for (h = 0; h < halves; ++h) {
                const int64_t o = out * halves + h;              /* output slot */
                float qe[3];
                int why;
                int32_t n;
                io.half = h;
                io.path = paths ? paths + o * path_stride * 3 : NULL;
                n = track_half(vol, prm, &io, &why, qe);
                /* SetEndPoint() */
                if (nsteps) nsteps[o] = n;
                if (reason) reason[o] = (uint8_t)why;
                if (end_xyz) for (a = 0; a < 3; ++a) end_xyz[o * 3 + a] = qe[a] + c[a];
            }
            /* count the streamlines passing through each target, once each */
            if (conn) {
                int t;
                for (t = 0; t < ntargets; ++t)
                    if (entered[t]) conn[si * ntargets + t] += 1u;
            }
            /* R25: each voxel the streamline passed through counts once (sort, then count
             * the distinct values) */
            if (umap) {
                int64_t k;
                qsort(entered_vox, (size_t)io.nentered, sizeof(int64_t), cmp_i64);
                for (k = 0; k < io.nentered; ++k)
                    if (k == 0 || entered_vox[k] != entered_vox[k - 1]) umap[entered_vox[k]] += 1u;
            }
        }
    }
    free(entered_vox);
    return 0;
}
