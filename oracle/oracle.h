/*
 * oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded CPU reference of the probabilistic-streamlining hot path
 * of Xu et al., "Probabilistic Brain Fiber Tractography on GPUs" (IPDPSW 2012).
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
 * --impl reference) may load it.  It shares no code, header or constant with the CUDA
 * path (paper_conf_ipps_xuzwrwxgxy12_b200/csrc, include/pt.h) and includes neither.
 *
 * Citations: P:Lnnn = line nnn of the paper text; Rnn = a reading of the
 * paper recorded in DESIGN.md "Readings".
 */
#ifndef ORACLE_H
#define ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Input volume in the canonical layout (Fig. 1: per-voxel sample volumes
 * of the fibre directions and fractions; directions given as Cartesian vectors, R20).
 *   dyads [F][S][Z][Y][X][3]  (x fastest, xyz innermost)
 *   f     [F][S][Z][Y][X]
 *   mask  [Z][Y][X]           (!= 0 inside)
 * is_half = 0: float32 values; 1: IEEE binary16 bit patterns (uint16). */
typedef struct {
    int32_t nx, ny, nz, nsamples, nfibres;
    int32_t is_half;
    const void* dyads;
    const void* f;
    const uint8_t* mask;
} oracle_volume;

/* step: step length in voxels (R3); curv_thr: continue iff |dot| > curv_thr (R4,
 * P:L117); fib_thr: fibre eligibility f_j > fib_thr (R7); max_steps (R14);
 * rng_seed: Philox key (R16); particles_per_seed P: pid = seed_id * P + j. */
typedef struct {
    float step, curv_thr, fib_thr;
    int32_t max_steps;
    uint64_t rng_seed;
    int64_t particles_per_seed;
    /* 0: a fresh random sample every step (R1, FSL style, the north star's mode);
     * 1: paper mode (NEXT-1): particle j of a seed follows sample volume j mod S for its
     *    whole path (Alg. 1: one sample volume per streamline). */
    int32_t sample_mode;
    /* NEXT-3 FSL-fidelity variants (R22-R24); all 0 = the north star's contract.
     * bidir: 1 = bidirectional streamlines (R22): half 0 is the one-directional particle,
     *        half 1 restarts at the seed with previous direction -d0 (d0 = half 0's first
     *        step direction) and draws from RNG stream 1.
     * interp: 1 = probabilistic (trilinear) interpolation of the sampled voxel (R23,
     *        "Interpolation()" P:L175), uniforms from RNG stream 2 + half.
     * init_fibre: first-step fibre of half 0 (R24): 0 = fibre 0 (R5), 1 = uniform among
     *        the eligible fibres, 2 = f-weighted among the eligible fibres. */
    int32_t bidir;
    int32_t interp;
    int32_t init_fibre;
} oracle_params;

enum { ORACLE_END_MASK = 0, ORACLE_END_CURV = 1, ORACLE_END_MAXLEN = 2 };

/* Philox4x32-10 (R16): one block, ctr[4], key[2] -> out[4]. */
void oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* binary16 -> float32, exact (R15). */
float oracle_half_to_float(uint16_t h);
void oracle_half_to_float_array(const uint16_t* h, float* out, int64_t n);
/* voxel index along one axis for a centred coordinate q (R10). */
int64_t oracle_axis_index(float q, int32_t n_axis);
/* sample index for a 32-bit word (R16): floor(w * S / 2^32). */
uint32_t oracle_sample_index(uint32_t w, uint32_t nsamples);

/* Track particles j in [j_begin, j_end) of every seed (Alg. 1 P:L159-187 inner loop with
 * the semantics of P:L98-121; contract "C-ALG" in DESIGN.md).
 *   seeds_xyz [nseeds][3] corner coordinates; seed_ids [nseeds] (NULL => 0..nseeds-1)
 *   map       [Z][Y][X] uint64, accumulated (+=) ; may be NULL
 *   nsteps, reason, end_xyz: per particle, index (seed_index*(j_end-j_begin) + j-j_begin);
 *                            each may be NULL.  With bidir, per half: index 2*that + half.
 *   paths     [particle][path_stride][3] corner-coordinate positions, point 0 = start,
 *             point k = after the k-th committed step, unused points = NaN; may be NULL
 *             (with bidir: [particle][2][path_stride][3], one polyline per half)
 *   labels    [Z][Y][X] target labels (0 = none, t+1 = target t) or NULL; ntargets <= 64
 *   conn      [nseeds][ntargets] uint64, accumulated: number of the seed's particles whose
 *             committed steps enter target t at least once (NEXT-2; R21); may be NULL
 *             (with bidir a streamline is the union of its two halves)
 *   umap      [Z][Y][X] uint64, accumulated: number of streamlines with at least one
 *             committed step landing in the voxel -- "counting the number of streamlines
 *             passing through B" (R25); may be NULL (with bidir a streamline is
 *             the union of its two halves)
 * Returns 0 on success, <0 on invalid arguments (nothing written). */
int oracle_track(const oracle_volume* vol, const oracle_params* prm,
                 const float* seeds_xyz, const uint64_t* seed_ids, int64_t nseeds,
                 int64_t j_begin, int64_t j_end,
                 uint64_t* map, int32_t* nsteps, uint8_t* reason, float* end_xyz,
                 float* paths, int32_t path_stride,
                 const uint8_t* labels, int32_t ntargets, uint64_t* conn, uint64_t* umap);


/* ---------------------------------------------------------------- NEXT-4: MCMC sampler
 * (oracle_mcmc.c) Metropolis-Hastings sampling of Eq. 1, readings
 * M1-M9 of DESIGN.md §12.  Parameters per voxel, in MH order:
 *   omega = (S0, d, sigma, f_1, theta_1, phi_1, ..., f_N, theta_N, phi_N),  NP = 3 + 3N. */
#define ORACLE_MCMC_MAX_MEAS 256

typedef struct {
    int32_t nx, ny, nz, nmeas;
    const float* dwi;     /* [nmeas][nz][ny][nx] (x fastest, measurement slowest; Fig. 1) */
    const float* bvals;   /* [nmeas] b-values (ms/um^2 units: b d ~ 1)                     */
    const float* bvecs;   /* [nmeas][3] unit gradient directions                          */
    const uint8_t* mask;  /* [nz][ny][nx] voxels to sample (!= 0)                          */
} oracle_dwi;

typedef struct {
    int32_t nfibres;      /* N of Eq. 1, 1..3 (the paper: 2)                        */
    int32_t burnin;       /* NumBurnIn (500 in the paper's example)                */
    int32_t nsamples;     /* NumSamples (50)                                        */
    int32_t interval;     /* L, the sample interval (2)                             */
    int32_t adapt_every;  /* K loops between proposal updates (Fig. 2; M8)                 */
    uint64_t rng_seed;    /* Philox key (M6)                                                */
    uint32_t fixed;       /* bit k: parameter k keeps its initial value (M9)                */
} oracle_mcmc_params;

/* Eq. 1 for one parameter vector: mu[i], i < n. */
void oracle_mcmc_signal(int nfibres, const double* omega, int n, const float* bvals,
                        const float* bvecs, double* mu);
/* The Gaussian and log-uniform of MH step (loop, voxel, k) (M6). */
void oracle_mcmc_draw(uint64_t seed, uint32_t loop, uint32_t voxel, uint32_t k, double* z,
                      double* logu);
/* Sample the voxels v in [v_begin, v_end) with mask != 0.
 *   init     [NP][V] initial states or NULL (automatic, M7)
 *   samples  [NP][nsamples][V] (written for sampled voxels only)
 *   accepted [NP][V] accepted proposals per parameter, or NULL
 * Returns 0, or < 0 for invalid arguments. */
int oracle_mcmc(const oracle_dwi* dw, const oracle_mcmc_params* p, const double* init,
                int64_t v_begin, int64_t v_end, double* samples, uint32_t* accepted);

#ifdef __cplusplus
}
#endif
#endif
