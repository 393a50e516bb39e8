/*
 * pt.h -- C ABI of the B200-native probabilistic-streamlining particle stepper.
 *
 * Method: Xu et al., "Probabilistic Brain Fiber Tractography on GPUs", IPDPS workshops
 * 2012.  Citations P:Lnnn are PAPER.md lines; Rnn are the readings of the
 * paper listed in DESIGN.md ("Readings").  The operations follow the paper's problem
 * statement: the user supplies the sample volumes of the fibre directions/fractions
 * (Fig. 1), start points, a step length and the termination criteria
 * (maximum angle, maximum steps); they get back fibre paths and/or
 * per-voxel visitation counts.
 *
 * Conventions for every entry point:
 *   - returns a pt_status; never throws or aborts across the ABI; the message of the
 *     last failure on a context is pt_last_error(ctx);
 *   - pointer arguments may be host or device pointers (detected with
 *     cudaPointerGetAttributes) unless stated otherwise; inputs are borrowed for the
 *     duration of the call (copied), outputs are caller-owned;
 *   - one context per (thread, GPU); distinct contexts are independent.
 *   - no torch types: plain pointers and sizes.  The Python binding passes
 *     tensor.data_ptr() and torch.cuda.current_stream().cuda_stream.
 */
#ifndef PT_H
#define PT_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct pt_ctx pt_ctx;

typedef enum {
    PT_OK = 0,
    PT_ERR_ARG = 1,       /* invalid argument (sizes, ranges, non-finite sample data) */
    PT_ERR_STATE = 2,     /* call out of order (e.g. pt_track before pt_load_samples) */
    PT_ERR_OOM = 3,       /* device allocation failed */
    PT_ERR_CUDA = 4,      /* CUDA runtime error; map contents are then unspecified */
    PT_ERR_OVERFLOW = 5   /* a uint32 map cell wrapped past 2^32-1 (R17) */
} pt_status;

typedef enum { PT_F32 = 0, PT_F16 = 1 } pt_dtype;

/* Termination reasons (P:L113-121 keeps max steps and max angle; R11 adds the mask). */
typedef enum { PT_END_MASK = 0, PT_END_CURV = 1, PT_END_MAXLEN = 2 } pt_reason;

/* pt_params.flags */
#define PT_REC_LEN        (1u << 0)  /* record per-particle nsteps (uint16)            */
#define PT_REC_REASON     (1u << 1)  /* record per-particle pt_reason (uint8)           */
#define PT_REC_END        (1u << 2)  /* record per-particle end point (3 x float32)     */
#define PT_REC_PATHS      (1u << 3)  /* record polylines, path_stride points/particle   */
#define PT_MAP_ACCUMULATE (1u << 4)  /* add to the map (and the connectivity matrix)
                                        instead of zeroing it first                     */
#define PT_REC_CONN       (1u << 5)  /* record the seed x target connectivity matrix for
                                        the targets of pt_load_targets (NEXT-2)          */
#define PT_KERNEL_SIMPLE  (1u << 8)  /* ablation: one thread per particle, no lane
                                        refill (the paper's "Extreme case 1")   */
#define PT_SEED_ORDER_INPUT (1u << 9) /* ablation: claim seeds in input order instead of
                                        the default Z-order (Morton) of their voxels;
                                        results are identical either way (R16)           */
#define PT_SAMPLE_PER_STREAMLINE (1u << 10) /* paper mode (NEXT-1): particle j of a seed
                                        follows sample volume j mod S for its whole path
                                        (Alg. 1) instead of a fresh
                                        random sample every step (R1)                    */
/* NEXT-3 FSL-fidelity variants (R22-R24; run by the variant kernel).        */
#define PT_BIDIR          (1u << 11) /* bidirectional streamlines (R22): each particle runs
                                        two halves from its seed; half 0 is the one-
                                        directional particle, half 1 starts against half
                                        0's first direction (RNG stream 1).  Per-particle
                                        outputs hold 2 entries per particle (index 2*i+h);
                                        the map counts both halves; a connectivity
                                        streamline is the union of the halves            */
#define PT_INTERP         (1u << 12) /* probabilistic (trilinear) interpolation of the
                                        sampled voxel, "Interpolation()" P:L175 (R23)    */
#define PT_INIT_RANDOM    (1u << 13) /* first fibre uniform over the eligible fibres (R24) */
#define PT_INIT_FWEIGHT   (1u << 14) /* first fibre drawn with probability f_j / sum f over
                                        the eligible fibres (R24); exclusive with
                                        PT_INIT_RANDOM                                   */
#define PT_KERNEL_VARIANT (1u << 15) /* run the variant kernel even with no variant flag
                                        (same results as the main kernel; ablation/tests) */
#define PT_KERNEL_SEGMENTED (1u << 16) /* ablation (ii): the paper's segmented relaunch
                                        (Table IV): one thread per live particle
                                        per segment of k steps, device stream compaction
                                        between segments, schedule of pt_set_segments.
                                        Same results; synchronous; not combinable with
                                        PT_REC_PATHS, PT_REC_CONN or the NEXT-3 variants */
#define PT_MAP_UNIQUE     (1u << 18) /* NEXT-2: the map counts streamlines, not steps: map[v]
                                        += 1 for every streamline (both halves of a
                                        bidirectional one together) with at least one
                                        committed step landing in voxel v ("counting
                                        the number of streamlines passing through B"; R25).
                                        Exact (a per-lane hash set of entered voxels).
                                        PT_ERR_ARG with PT_KERNEL_SIMPLE / SEGMENTED       */

/* Create a context on CUDA device `cuda_device` (the caller's current device is left
 * unchanged).  *out receives the context or NULL.  The stream defaults to the legacy
 * default stream until pt_set_stream. */
pt_status pt_create(int cuda_device, pt_ctx** out);
/* Free every device buffer of the context. NULL-safe. */
void pt_destroy(pt_ctx* ctx);
/* Message of the last failed call on ctx ("" if none); valid until the next call.
 * pt_last_error(NULL) returns the message of the last failed pt_create. */
const char* pt_last_error(const pt_ctx* ctx);
/* Stream (a cudaStream_t, or NULL for the legacy default stream) on which every later
 * call on ctx enqueues its work. */
pt_status pt_set_stream(pt_ctx* ctx, void* cuda_stream);

/* Sample volume shape: nx, ny, nz > 0; nsamples S >= 1 (the number of MCMC samples per
 * voxel); nfibres F in [1, 3] (N = 2 in the paper, Eq. 1);
 * dtype of the dyads/f arrays. */
typedef struct {
    int32_t nx, ny, nz, nsamples, nfibres;
    int32_t dtype; /* pt_dtype */
} pt_volume;

/* Load the per-voxel orientation samples (the six sample volumes f1,f2,theta1,theta2,
 * phi1,phi2 of P:L125, with (theta, phi) given as Cartesian unit vectors, R20) and the
 * tracking mask, and repack them on the device into one record per (voxel, sample).
 * The device records are voxel-major and BRICKED: the volume is cut into bricks of
 * 2^b x 2^b x 2^b voxels (b from the environment variable PT_BRICK: 4, the default, or 0 = plain
 * raster order; any other value is PT_ERR_ARG), so the records of a 3-D neighbourhood
 * are contiguous.
 * The layout is internal: it changes no result, only the padded device footprint
 * (ceil(n/2^b)*2^b per axis x S x record bytes; for volumes of <= 4 GB of records, one
 * more brick of sentinel records on every side of every axis, so that the tracking
 * kernel needs no bounds test per step; the largest |vector component| is recorded for
 * that bound).
 *   dyads: [F][S][nz][ny][nx][3] (x fastest, xyz innermost), float32 or binary16 bits
 *   f    : [F][S][nz][ny][nx], same dtype
 *   mask : [nz][ny][nx] uint8, != 0 inside
 * Host or device pointers; copied; the caller keeps ownership.  Replaces any previously
 * loaded volume.  Errors: PT_ERR_ARG for bad shapes, NULL pointers or a non-finite
 * dyad / f value inside the mask; PT_ERR_OOM; PT_ERR_CUDA.  Synchronises ctx's stream. */
pt_status pt_load_samples(pt_ctx* ctx, const pt_volume* vol, const void* dyads,
                          const void* f, const uint8_t* mask);

/* Tracking parameters (Sec. III-B3; Table II P:L283-291 uses step 0.1-0.3,
 * dot thresholds 0.8-0.9 and 50 samples). */
typedef struct {
    float step;                 /* step length in voxels, > 0 (R3)                       */
    float curv_thr;             /* continue iff |v . d_prev| > curv_thr, |curv_thr| <= 1
                                   (maximum angle "measured by the dot product"; R4) */
    float fib_thr;              /* fibre j eligible for the direction choice iff f_j > fib_thr (R7) */
    int32_t max_steps;          /* 1..65535 (maximum number of steps; R14)        */
    uint64_t rng_seed;          /* Philox-4x32-10 key (R16)                               */
    int64_t particles_per_seed; /* P >= 1; particle j of seed id k has pid = k*P + j      */
    uint32_t flags;             /* PT_REC_* | PT_MAP_ACCUMULATE | PT_MAP_UNIQUE |
                                   PT_KERNEL_SIMPLE | PT_KERNEL_SEGMENTED |
                                   PT_SEED_ORDER_INPUT | PT_SAMPLE_PER_STREAMLINE |
                                   PT_BIDIR | PT_INTERP | PT_INIT_* | PT_KERNEL_VARIANT   */
    int32_t path_stride;        /* points stored per particle with PT_REC_PATHS (>= 1)    */
} pt_params;

/* Track P particles from each seed (Algorithm 1, with the stepping
 * semantics of P:L98-121 and contract C-ALG of DESIGN.md).
 *   seeds_xyz: [nseeds][3] float32 corner-convention voxel coordinates (the centre of
 *              voxel i is i + 0.5)
 *   seed_ids : [nseeds] uint64 global seed ids, or NULL for 0..nseeds-1.  The RNG is
 *              keyed by pid = seed_id*P + j, so results do not depend on sharding or on
 *              the order of the seeds.
 *   map      : [nz][ny][nx] uint32 visitation counts (one per committed step at the new
 *              voxel, R13), zeroed first unless PT_MAP_ACCUMULATE; may be NULL.
 * The kernels count into a context-owned scratch map (a permuted and/or record-ordered
 * copy: one uint32 per padded record voxel, rounded up to a power of two when permuted)
 * that pt_track adds into `map` after the kernel;
 * `map` itself always receives raster-ordered counts.
 * With device pointers the call is asynchronous on ctx's stream; a host `map` makes it
 * synchronous (device map, then a device-to-host copy).  Per-particle outputs selected
 * by flags stay on the device until pt_get_paths.  Errors: PT_ERR_STATE before
 * pt_load_samples; PT_ERR_ARG for parameter ranges, nseeds < 0 or pid overflow;
 * PT_ERR_OOM; PT_ERR_CUDA; PT_ERR_ARG for PT_KERNEL_SIMPLE combined with a NEXT-3
 * variant flag or for PT_INIT_RANDOM | PT_INIT_FWEIGHT.  Map overflow is reported by
 * pt_get_stats/pt_get_paths. */
pt_status pt_track(pt_ctx* ctx, const float* seeds_xyz, const uint64_t* seed_ids,
                   int64_t nseeds, const pt_params* params, uint32_t* map);

/* Segment schedule of PT_KERNEL_SEGMENTED: NumIteration[] of the paper,
 * intervals[0..n-1] steps per segment, the last one repeating until no particle is alive.
 * Default: strategy B = {1, 2, 5, 10, 20, 50, 100, 200, 500}.  Errors: PT_ERR_ARG for
 * n < 1, n > 64 or an interval < 1. */
pt_status pt_set_segments(pt_ctx* ctx, const int32_t* intervals, int32_t n);

/* Target regions for the seed x target connectivity matrix (NEXT-2; the connectivity
 * estimate of P:L109, "counting the number of streamlines passing through B, and dividing
 * it by the total number", with B a labelled region).
 *   labels  : [nz][ny][nx] uint8 of the loaded volume's shape, 0 = no target, t in
 *             1..ntargets = target t-1.  Host or device; copied.  NULL (or ntargets 0)
 *             removes the targets.
 *   ntargets: 0..64.
 * Errors: PT_ERR_STATE before pt_load_samples; PT_ERR_ARG for ntargets > 64. */
pt_status pt_load_targets(pt_ctx* ctx, const uint8_t* labels, int32_t ntargets);

/* Seed x target matrix of the last pt_track with PT_REC_CONN: out[s][t] (uint32) = number
 * of seed s's particles whose path (the voxels of its committed steps, R13/R21) enters
 * target t at least once; s = seed index of that call.  capacity = elements out holds
 * (>= nseeds * ntargets, else PT_ERR_ARG); *count receives nseeds * ntargets (query with
 * out = NULL).  Host or device out; synchronises ctx's stream. */
pt_status pt_get_connectivity(pt_ctx* ctx, uint32_t* out, int64_t capacity, int64_t* count);

/* Per-particle outputs of the last pt_track, particle index = seed_index*P + j
 * (with PT_BIDIR: entry 2*(seed_index*P + j) + half, count = 2 * nseeds * P).
 * Set capacity = number of particles the buffers hold; NULL buffers are skipped;
 * count receives the number of particles of the last pt_track (query with all buffers
 * NULL).  nsteps [count] uint16; reason [count] uint8; end_xyz [count][3] float32
 * corner coordinates; paths [count][path_stride][3] float32 (point 0 = start, point k =
 * after the k-th committed step, unused points NaN).  Requesting an output that the
 * last pt_track did not record is PT_ERR_STATE; capacity < count is PT_ERR_ARG.
 * Synchronises ctx's stream; returns PT_ERR_OVERFLOW if the map wrapped.  Paper: the
 * fibre paths of Fig. 1 and the end points of Alg. 1 (SetEndPoint() /
 * ReadEndPointFromGPU()). */
typedef struct {
    uint16_t* nsteps;
    uint8_t* reason;
    float* end_xyz;
    float* paths;
    int64_t capacity;
    int64_t count;       /* out */
    int32_t path_stride; /* out */
} pt_paths;
pt_status pt_get_paths(pt_ctx* ctx, pt_paths* out);

/* Counters of the last pt_track (synchronises ctx's stream).
 *   total_steps      : sum of nsteps over all particles (= sum of the map, R13)
 *   particles        : particles tracked
 *   lane_active      : sum over warp step-iterations of live lanes
 *   lane_slots       : 32 x warp step-iterations (active-lane fraction = ratio)
 *   map_sum          : sum of the map cells after the call (mod 2^64)
 *   overflow         : 1 if a map cell wrapped (detected as map_sum != expected)
 *   kernel_ms        : device time of the tracking kernel (CUDA events on ctx's stream)
 *   track_ms         : device time of the whole pt_track enqueue (zeroing, kernel, checks)
 *   unique_visits    : with PT_MAP_UNIQUE, the counts added to the map (sum over
 *                      streamlines of the voxels they entered); else 0
 * Errors: PT_ERR_OVERFLOW (see overflow); PT_ERR_ARG if a device-resident seed id made
 * seed_id*P + j overflow 64 bits (those particles ran with seed id 0). */
typedef struct {
    uint64_t total_steps;
    uint64_t particles;
    uint64_t lane_active;
    uint64_t lane_slots;
    uint64_t map_sum;
    int32_t overflow;
    float kernel_ms;
    float track_ms;
    uint64_t unique_visits;
} pt_stats;
pt_status pt_get_stats(pt_ctx* ctx, pt_stats* out);

/* Timing of the last pt_load_samples (the paper's Copy3DImagesToGPU(), timed as
 * "Transfer" in Table II): device time of the host-to-device copies of the host inputs
 * (0 if every input was a device pointer) and of the repack kernel, bytes copied from the
 * host, bytes of the repacked record volume.  Errors: PT_ERR_STATE before a load. */
typedef struct {
    float h2d_ms;
    float repack_ms;
    uint64_t h2d_bytes;
    uint64_t record_bytes;
} pt_load_stats;
pt_status pt_get_load_stats(pt_ctx* ctx, pt_load_stats* out);

/* Device self-test of the tracking RNG (R16): for i < n,
 * words[4i..4i+3] = Philox4x32-10(ctr = {block[i], lo32(pid[i]), hi32(pid[i]), stream[i]},
 * key = {lo32(rng_seed), hi32(rng_seed)}) and samples[3i+k] = floor(words[4i+k] * nsamples
 * / 2^32), k < 3, computed by the SAME device functions the tracking kernel uses; the
 * kernel also recomputes each block with the CUDA library's curand_Philox4x32_10 and
 * *mismatches receives the number of blocks that differ (0 expected).  All arrays host or
 * device; nsamples >= 1.  Synchronous.  Errors: PT_ERR_ARG for NULL arrays / n < 0. */
pt_status pt_rng_draws(pt_ctx* ctx, const uint64_t* pid, const uint32_t* block, const uint32_t* stream,
                       int64_t n, uint64_t rng_seed, uint32_t nsamples, uint32_t* words, uint32_t* samples,
                       int64_t* mismatches);

/* Roofline micro-benchmark: uniformly random, record-aligned
 * reads of `record_bytes` (8, 16, 32 or 64) from a device buffer of `buffer_bytes`,
 * full occupancy, no other work.  *sectors_per_s receives 32-byte sectors per second.
 * Synchronous. */
pt_status pt_gather_bench(pt_ctx* ctx, int64_t buffer_bytes, int32_t record_bytes,
                          double* sectors_per_s);

/* Record bytes of the repacked layout for (nfibres, dtype): 16/32/64 (f32) or 8/16/32
 * (f16).  Returns 0 for invalid arguments. */
int32_t pt_record_bytes(int32_t nfibres, int32_t dtype);


/* ===================================================================================
 * NEXT-4: MCMC sampling of the local fibre model (the paper's first GPU step, Sec. III-A
 * P:L61-90, Sec. IV-A and Fig. 2; contract C-MCMC and readings M1-M9 of
 * DESIGN.md §12).  Per valid voxel, Metropolis-Hastings on Eq. 1 (the multiple partial
 * volume model) with parameters, in MH order,
 *     omega = (S0, d, sigma, f_1, theta_1, phi_1, ..., f_N, theta_N, phi_N),  NP = 3 + 3N.
 * Arithmetic is binary64.  The sample volumes (f_j, theta_j, phi_j) feed pt_load_samples
 * through pt_mcmc_to_volume (Fig. 1).
 * =================================================================================== */
typedef struct {
    int32_t nx, ny, nz;   /* volume                                                        */
    int32_t nmeas;        /* n: measurements per voxel, 1..128                               */
} pt_dwi_shape;

typedef struct {
    int32_t nfibres;      /* N of Eq. 1, 1..3 (the paper: 2)                          */
    int32_t burnin;       /* NumBurnIn >= 0 (500)                                     */
    int32_t nsamples;     /* NumSamples >= 1 (50)                                     */
    int32_t interval;     /* L >= 1, the sample interval (2)                          */
    int32_t adapt_every;  /* K >= 1: loops between proposal updates (Fig. 2; M8: 50)          */
    uint64_t rng_seed;    /* Philox key (M6)                                                  */
    uint32_t fixed;       /* bit k: parameter k keeps its initial value (M9); bits >= NP = 0  */
} pt_mcmc_params;

/* Run the sampler on every voxel with mask != 0.
 *   dwi     : [nmeas][nz][ny][nx] float32 (the 4-D volume of Fig. 1, measurement slowest)
 *   bvals   : [nmeas] float32 b-values;  bvecs: [nmeas][3] float32 unit gradient directions
 *   mask    : [nz][ny][nx] uint8, the voxels to sample ("valid (white matter)" voxels)
 *   init    : [NP][nz][ny][nx] float64 initial states, or NULL for the automatic initial
 *             state (M7)
 *   samples : [NP][nsamples][nz][ny][nx] float64 out (host or device; voxels outside the
 *             mask are set to 0)
 *   accepted: [NP][nz][ny][nx] uint32 out: accepted proposals per parameter, or NULL
 * Inputs host or device (copied / read in place); synchronous.  Errors: PT_ERR_ARG for
 * shapes, nmeas > 128, nfibres outside 1..3, burnin + nsamples*interval >= 2^32, NULL
 * pointers; PT_ERR_OOM; PT_ERR_CUDA. */
pt_status pt_mcmc(pt_ctx* ctx, const pt_dwi_shape* shape, const float* dwi, const float* bvals,
                  const float* bvecs, const uint8_t* mask, const pt_mcmc_params* params,
                  const double* init, double* samples, uint32_t* accepted);

/* Counters of the last pt_mcmc (synchronises): voxels sampled, MH steps attempted
 * (voxels x loops x free parameters), proposals accepted, kernel time (CUDA events). */
typedef struct {
    uint64_t voxels;
    uint64_t mh_steps;
    uint64_t accepted;
    float kernel_ms;
} pt_mcmc_stats;
pt_status pt_get_mcmc_stats(pt_ctx* ctx, pt_mcmc_stats* out);

/* Convert pt_mcmc samples into the tracker's canonical sample volumes (R20: the (theta,
 * phi) -> unit vector conversion happens here, outside both trackers):
 *   samples: [3+3N][S][nz][ny][nx] float64 (device or host)
 *   dyads  : [N][S][nz][ny][nx][3] float32 out = (sin th cos ph, sin th sin ph, cos th)
 *   f      : [N][S][nz][ny][nx] float32 out
 * Voxels with mask == 0 get zeros.  Output device or host; synchronous. */
pt_status pt_mcmc_to_volume(pt_ctx* ctx, const pt_dwi_shape* shape, int32_t nfibres,
                            int32_t nsamples, const double* samples, const uint8_t* mask,
                            float* dyads, float* f);

#ifdef __cplusplus
}
#endif
#endif
