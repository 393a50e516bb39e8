// pt_internal.h -- private interface between the C-ABI host code (pt_api.cu) and the
// kernels (pt_kernels.cu).  Not installed; not part of include/pt.h.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace pt {

#ifndef PT_CTA_THREADS
#define PT_CTA_THREADS 1024
#endif
// Persistent kernel: one CTA of kThreads per SM; a CTA claims a chunk of cta_chunk particles
// of one seed per global atomic (cta_chunk chosen per call, see pt_track: a whole seed when
// there is enough work) and hands kSub-particle sub-chunks to its warps (shared-memory
// tickets), so a seed's particles run on one SM (L1 locality) while the chip as a whole
// works on a compact set of Morton-adjacent seeds (L2 locality).
constexpr int kThreads = PT_CTA_THREADS;
constexpr int kSimpleThreads = 256;  // no-refill ablation kernel
#ifndef PT_CTA_THREADS_EXT
#define PT_CTA_THREADS_EXT 768
#endif
constexpr int kThreadsExt = PT_CTA_THREADS_EXT;  // variant / unique-map instantiations
// Permuted scratch map (map_mask != 0): the kernels count into a scratch map whose cell of
// voxel v keeps the low PT_MAP_GRAN bits of v and multiplies the rest by an odd constant
// mod 2^k (a bijection on [0, 2^(k+g)) >= V), so the RED bursts of the compact neighbourhood
// the CTAs work on spread over all L2 slices instead of a few; pt_track then adds the
// scratch into the caller's raster map (map_unpermute).
#ifndef PT_MAP_PERM
#define PT_MAP_PERM 1  // 0: never permute; 1: permute when the record volume is <= PT_BIG_VOLUME; 2: always
#endif
#ifndef PT_MAP_GRAN
#define PT_MAP_GRAN 0  // log2 voxels kept together per permuted unit
#endif
constexpr uint32_t kMapMul = 0x9E3779B1u;
__host__ __device__ __forceinline__ uint32_t map_perm(uint32_t v, uint32_t mask) {
    constexpr uint32_t g = PT_MAP_GRAN, lo = (1u << g) - 1u;
    return ((((v >> g) * kMapMul) & mask) << g) | (v & lo);
}
constexpr uint32_t kSub = 32;
constexpr uint32_t kMinCtaChunk = 1024;

// Indices of the per-call device counters (unsigned long long[kNumStats]).
enum StatIdx {
    kStatSteps = 0,      // sum of nsteps
    kStatParticles = 1,  // particles finished
    kStatLaneActive = 2, // live lanes summed over warp step-iterations
    kStatLaneSlots = 3,  // 32 x warp step-iterations
    kStatMapAfter = 4,   // sum of map cells after the kernel
    kStatMapBefore = 5,  // sum of map cells before the kernel (accumulate mode)
    kStatQueue = 6,      // work-queue counter (chunks claimed)
    kStatBadInput = 7,   // repack: non-finite value inside the mask
    kStatBadId = 8,      // a device-resident seed id whose pid overflows 64 bits
    kStatUnique = 9,     // UNQ: first entries counted (= increments of the unique map)
    kStatLabelMax = 10,  // pt_load_targets: largest label
    kStatBadAccess = 11, // PT_CHECK_BOUNDS builds: a device access outside its buffer
    kStatMaxAbs = 12,    // repack: bits of the largest |vector component| inside the mask
    kNumStats = 13
};

// Bounds-checked build (-DPT_CHECK_BOUNDS=1, tests/test_gpu_bounds.py): every record gather,
// map / hash-set / mask / label / output access of the tracking kernels is checked against
// the size of its buffer (TrackArgs::*_n); a violation sets stats[kStatBadAccess] and
// pt_get_stats fails.  Replaces compute-sanitizer memcheck, which this GPU pool does not run.
#ifndef PT_CHECK_BOUNDS
#define PT_CHECK_BOUNDS 0
#endif
#if PT_CHECK_BOUNDS
#define PT_BOUND(a, cond)                                                                          \
    do {                                                                                         \
        if (!(cond)) atomicOr((a).stats + ::pt::kStatBadAccess, 1ull);                           \
    } while (0)
#else
#define PT_BOUND(a, cond) \
    do {                  \
    } while (0)
#endif

struct TrackArgs {
    const uint8_t* rec;          // [V'][S] records of rec_bytes, voxel order rec_vox() (bricked)
    uint32_t rb_log, rb_nbx, rb_nby;  // record layout: brick edge 2^rb_log (0 or kBrickLog), bricks per row / column
    uint32_t rb_ky, rb_kz;       // per-axis brick strides minus the shifted part (PT_REC_AFFINE)
    uint32_t rb_off;             // margin offset of the voxel coordinates (RecLayout::off)
    int pcx, pcy, pcz;           // cx + rb_off etc.: padded coordinates straight from the lookup
    uint32_t nobounds;           // 1: the margin covers every candidate (step * max|v| < rb_off)
    int nx, ny, nz;
    int cx, cy, cz;              // floor(N/2) per axis
    float fcx, fcy, fcz;         // the same as floats
    uint32_t S;
    uint32_t sample_mode;        // 0: random sample per step (R1); 1: s = j mod S (NEXT-1)
    float step, curv_thr, fib_thr;
    int max_steps;
    uint32_t key0, key1;
    uint64_t P;                  // particles per seed
    const float* seeds;          // [nseeds][3] corner coordinates
    const uint64_t* seed_ids;    // [nseeds] or nullptr
    const uint32_t* order;       // [nseeds] processing order (Morton) or nullptr
    uint64_t nseeds;
    uint64_t nparticles;         // nseeds * P
    uint32_t cta_chunk;          // particles per CTA claim within a seed (multiple of kSub)
    uint32_t seeds_per_claim;    // > 1: a claim is this many whole consecutive seeds ...
    uint64_t group_chunks;       // ... for claims < group_chunks; later claims are one seed each
    uint32_t chunks_per_seed;    // ceil(P / cta_chunk)
    uint64_t total_chunks;       // nseeds * chunks_per_seed
    uint64_t max_seed_id;        // largest seed id whose pids fit 64 bits: (2^64-1 - (P-1)) / P
    uint32_t* map;               // [V] raster map this launch adds into, or nullptr
    uint16_t* o_nsteps;          // [nparticles] or nullptr
    uint8_t* o_reason;
    float* o_end;                // [nparticles][3]
    float* o_paths;              // [nparticles][path_stride][3]
    const uint8_t* labels;       // [V] target labels (0 none, t+1) or nullptr
    uint32_t ntargets;
    uint32_t* conn;              // [nseeds][ntargets] seed x target matrix or nullptr
    int path_stride;
    unsigned long long* stats;   // [kNumStats]
    // NEXT-3 variants (VAR instantiations only; R22-R24)
    uint32_t bidir;              // 1: two halves per particle, outputs at 2*i + half
    uint32_t interp;             // 1: probabilistic interpolation of the sampled voxel
    uint32_t init_mode;          // first fibre: 0 fibre 0, 1 uniform eligible, 2 f-weighted
    const uint8_t* mask;         // [V] tracking mask (interp: candidate test) or nullptr
    // NEXT-2 per-streamline-unique map (UNQ instantiations only; R25)
    unsigned long long* utab;    // [lanes][2^ulog] generation-tagged hash sets, zeroed per call
    uint32_t ulog;               // log2 entries per lane's hash set
    uint64_t max_ctas;           // CTAs the hash-set buffer covers
    // buffer sizes, read only by PT_CHECK_BOUNDS builds
    uint64_t rec_n;              // records in rec (allocated voxels x S)
    uint64_t V;                  // voxels of map / mask / labels (nx ny nz)
    uint64_t out_n;              // entries of o_nsteps / o_reason / o_end (particles x halves)
    uint32_t utab_lanes;         // lanes (hash sets) in utab
    uint32_t map_mask;           // 0: raster map; else permuted units of the scratch map - 1
    int32_t fib_h;               // fp16 records, fib_thr >= 0: (smallest binary16 > fib_thr) << 16
    uint64_t map_keys;           // map keys: V (raster voxel) or the padded record voxels (rv keys)
};
// cell of voxel v in the map the kernels add into
__host__ __device__ __forceinline__ uint32_t map_cell(const TrackArgs& a, uint32_t v) {
    return a.map_mask ? map_perm(v, a.map_mask) : v;
}

// Which instantiation of the tracking kernel a call runs.
struct TrackMode {
    bool simple;  // no-refill ablation (i)
    bool out;     // per-particle outputs / polylines / connectivity recorded
    bool var;     // NEXT-3 variants (run-time selected by bidir / interp / init_mode)
    bool unique;  // NEXT-2 per-streamline-unique map
};


// NEXT-4 MCMC sampler (pt_mcmc.cu): one warp per voxel of the compacted mask list.
enum McmcStatIdx { kMcmcStatAccepted = 0, kMcmcStatBadAccess = 1, kMcmcNumStats = 2 };  // 1: PT_CHECK_BOUNDS
struct McmcArgs {
    const float* dwi;            // [nmeas][V]
    const float* bvals;          // [nmeas]
    const float* bvecs;          // [nmeas][3]
    const uint32_t* vox;         // [nvox] linear indices of the mask voxels
    uint32_t nvox;
    uint32_t* queue;             // voxel work counter (zeroed per call)
    uint64_t V;
    int nmeas, nfibres;
    uint32_t burnin, nsamples, interval, adapt_every, loops;
    uint32_t key0, key1;
    uint32_t fixed;              // bit k: parameter k held at its initial value (M9)
    const double* init;          // [NP][V] or nullptr (automatic initial state, M7)
    double* samples;             // [NP][nsamples][V]
    uint32_t* accepted;          // [NP][V] or nullptr
    unsigned long long* stats;   // [kMcmcNumStats]
};
size_t mcmc_select_temp_bytes(uint64_t V);
cudaError_t launch_mcmc_voxel_list(const uint8_t* mask, uint64_t V, uint8_t* flags, uint32_t* out, uint32_t* nsel,
                                   void* temp, size_t temp_bytes, cudaStream_t st);
cudaError_t launch_mcmc(const McmcArgs& a, int num_sms, cudaStream_t st);
cudaError_t launch_samples_to_volume(const double* samples, const uint8_t* mask, uint64_t V, int N, int S,
                                     float* dyads, float* f, cudaStream_t st);

// Ablation (ii): segmented relaunch with device compaction (pt_segmented.cu).  State of a
// batch of particles, SoA; live / flag are indexed by list position.
struct SegState {
    float* q;        // [batch][3] position (centred)
    float* p;        // [batch][3] previous direction
    uint32_t* n;     // [batch] committed steps
    uint32_t* vox;   // [batch] voxel of q
    uint64_t* pid;   // [batch] RNG particle id
    uint64_t* li;    // [batch] output index (seed index * P + j)
    uint32_t* live;  // [batch] live list (identity after init)
    uint8_t* flag;   // [batch] alive flag per list position
};
size_t seg_select_temp_bytes(uint32_t n);
cudaError_t run_segmented(const TrackArgs& a, int F, bool half, const SegState& s, uint32_t batch,
                          const int32_t* schedule, int nsched, uint32_t* live_b, uint32_t* d_count, void* temp,
                          size_t temp_bytes, cudaStream_t st);

// Launchers (return the launch error, if any).  launch_track dispatches on (F, precision)
// to launch_track_f<F, HALF> (pt_track_f<F>_<f32|f16>.cu, one translation unit each).
cudaError_t launch_track(const TrackArgs& a, const TrackMode& m, int nfibres, bool half, int num_sms,
                         cudaStream_t st);
template <int F, bool HALF>
cudaError_t launch_track_f(const TrackArgs& a, const TrackMode& m, int num_sms, cudaStream_t st);
// pt_rng_draws: the tracking RNG on explicit counters, cross-checked against curand
cudaError_t launch_rng_draws(const uint64_t* pid, const uint32_t* block, const uint32_t* stream, int64_t n,
                             uint32_t k0, uint32_t k1, uint32_t S, uint32_t* words, uint32_t* samples,
                             unsigned long long* mismatches, cudaStream_t st);
// max over the target labels (pt_load_targets validation) into *out
cudaError_t launch_label_max(const uint8_t* labels, int64_t V, unsigned long long* out, cudaStream_t st);
// Record layout (see rec_vox in pt_device.cuh): b = brick log2 edge, 0 (raster) or
// kBrickLog (the default; the main tracking kernel is compiled for these two).
constexpr uint32_t kBrickLog = 4;
// PT_REC_MARGIN: bricked layouts get one brick of sentinel records on every side (the
// voxel coordinates are offset by off = 2^b), so a candidate up to 2^b voxels outside the
// volume reads a sentinel record: the bench instantiation needs no bounds test per step.
#ifndef PT_REC_MARGIN
#define PT_REC_MARGIN 1
#endif
struct RecLayout {
    uint32_t b, nbx, nby, nbz;
    uint32_t off = 0;  // coordinate offset of the volume inside the brick grid (margin)
    uint64_t nvox() const { return (uint64_t)nbx * nby * nbz << (3u * b); }  // allocated voxels (padded)
};
RecLayout rec_layout(int nx, int ny, int nz, uint32_t b, bool margin);
cudaError_t launch_repack(const void* dyads, const void* f, const uint8_t* mask, uint8_t* rec,
                          int nx, int ny, int nz, const RecLayout& L, int S, int F, bool half, int rec_bytes,
                          unsigned long long* bad, unsigned long long* maxabs, cudaStream_t st);
// Z-order processing permutation of the seeds: perm[k] = index of the k-th seed in Morton
// order of its voxel (ties by input index; stable radix sort).  keys, keys_out, idx, perm:
// device buffers of nseeds; temp: seed_order_temp_bytes(nseeds) bytes.
size_t seed_order_temp_bytes(uint64_t nseeds);
cudaError_t launch_seed_order(const float* seeds, uint64_t nseeds, uint32_t* keys, uint32_t* keys_out,
                              uint32_t* idx, uint32_t* perm, void* temp, size_t temp_bytes, cudaStream_t st);
cudaError_t launch_map_sum(const uint32_t* map, int64_t V, unsigned long long* out,
                           cudaStream_t st);
// map[v] (+)= scratch[cell(key(v))]: key = v or its record voxel rv (RecLayout L), cell =
// map_perm(key, mask) or key (mask 0)
cudaError_t launch_map_unpermute(const uint32_t* scratch, uint32_t mask, bool rv_keys, int nx, int ny,
                                 const RecLayout& L, uint32_t* map, int64_t V, bool accumulate, cudaStream_t st);
cudaError_t launch_gather_bench(const uint8_t* buf, uint64_t nrec, int rec_bytes, uint32_t iters,
                                int blocks, uint32_t seed, uint32_t* sink, cudaStream_t st);
int gather_bench_blocks_per_sm(int rec_bytes);

// The bench instantiations (compile-time bricked record layout, no outputs, default
// semantics) key the map by the record voxel rv their gathers already computed (no raster
// index per step); every other instantiation by the raster voxel.  pt_track sizes and
// reads back the scratch map accordingly; launch_track_fh takes the same decision.
#ifndef PT_RVKEYS
#define PT_RVKEYS 1  // 0: every instantiation keys the map by raster voxel (A/B switch)
#endif
inline bool track_rv_keys(const TrackArgs& a, const TrackMode& m, bool half) {
    return PT_RVKEYS && !m.simple && !m.unique && !m.var && !m.out && !a.sample_mode &&
           !(half && !(a.fib_thr >= 0.f)) && a.rb_log == kBrickLog;
}

}  // namespace pt
