// pt_api.cu -- host side of the C ABI declared in include/pt.h.
//
// Owns the device state of one context: the repacked record volume, per-call particle
// outputs, counters and CUDA events.  Every call enqueues on the context's stream and
// converts CUDA failures into pt_status codes with a message (no exceptions cross the ABI).
#include "pt.h"

#include <cuda_runtime.h>

#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "pt_internal.h"

#ifndef PT_SEEDS_PER_CLAIM
// Whole seeds per CTA claim when every seed fits one claim: a CTA walks G consecutive
// (Morton-adjacent) seeds, so its L1 keeps serving the shared tract voxels, while the
// chip-wide span of in-flight seeds (#SMs x G) sets the L2 working set.  Round 1 (raster
// map) preferred G = 32 on c3 / c4 (sweep 1..64: 74.6 ... 77.2 G); once the map REDs were
// spread over the L2 slices (permuted scratch map, r02n) the L2 side dominates: G = 1 / 2 /
// 4 / 8 / 16 / 32 give c3 161.9 / 163.7 / 163.5 / 161.1 / 155.4 / 146.8 G, c4 (half the
// record bytes) peaks at G = 8-12 (185.5-186.2 G), c5 at 4 (97.9 G)
// (profiles/r02y_claims_ab.log, r02z_claims_sweep.log, r02aa_claims_small.log): G = 8 for
// record payloads up to PT_SMALL_VOLUME bytes, else 4.
#define PT_SEEDS_PER_CLAIM 8
#endif
#ifndef PT_SEEDS_PER_CLAIM_BIG
#define PT_SEEDS_PER_CLAIM_BIG 4
#endif
#ifndef PT_SMALL_VOLUME
#define PT_SMALL_VOLUME (1ull << 30)
#endif
#ifndef PT_BIG_VOLUME
#define PT_BIG_VOLUME (4ull << 30)
#endif
#ifndef PT_TAIL_SEEDS_PER_SM
#define PT_TAIL_SEEDS_PER_SM 4  // single-seed claims at the end of the queue, per SM
#endif
#ifndef PT_BRICK_DEFAULT
#define PT_BRICK_DEFAULT 4  // record layout brick log2 edge (0 = raster, 4 = 16^3 bricks, measured best)
#endif

struct pt_ctx {
    int device = 0;
    int num_sms = 0;
    cudaStream_t stream = nullptr;
    std::string err;
    // volume
    bool loaded = false;
    pt_volume vol{};
    int rec_bytes = 0;
    pt::RecLayout layout{};       // record voxel order (bricked, rec_vox)
    float max_abs = 0.f;          // largest |vector component| inside the mask (margin test)
    uint8_t* d_rec = nullptr;
    size_t rec_size = 0;
    uint64_t rec_payload = 0;     // V x S x record bytes (the size rules below use this, not the padded size)
    uint8_t* d_mask = nullptr;    // tracking mask copy (the variant kernel's interpolation)
    size_t mask_cap = 0;
    // per-call buffers
    float* d_seeds = nullptr;
    size_t seeds_cap = 0;
    uint64_t* d_ids = nullptr;
    size_t ids_cap = 0;
    uint32_t* d_order = nullptr;  // seed order: 4 x nseeds u32 (keys, sorted keys, idx, perm)
    size_t order_cap = 0;
    uint8_t* d_temp = nullptr;    // radix-sort temp storage
    size_t temp_cap = 0;
    uint32_t* d_map = nullptr;   // internal map for host map pointers
    size_t map_cap = 0;
    uint32_t* d_pmap = nullptr;  // PT_MAP_PERM: permuted scratch map
    size_t pmap_cap = 0;
    unsigned long long* d_utab = nullptr;  // NEXT-2 unique map: per-lane hash sets
    size_t utab_cap = 0;
    uint8_t* d_stage = nullptr;    // pt_load_samples: staging of host inputs (grow-only)
    size_t stage_cap = 0;
    cudaEvent_t lev[3] = {nullptr, nullptr, nullptr};  // load: start, after H2D, after repack
    uint64_t load_h2d_bytes = 0;
    uint16_t* d_nsteps = nullptr;
    size_t nsteps_cap = 0;
    uint8_t* d_reason = nullptr;
    size_t reason_cap = 0;
    float* d_end = nullptr;
    size_t end_cap = 0;
    float* d_paths = nullptr;
    size_t paths_cap = 0;
    unsigned long long* d_stats = nullptr;
    uint8_t* d_labels = nullptr;   // NEXT-2 target labels [V]
    size_t labels_cap = 0;
    int32_t ntargets = 0;
    uint32_t* d_conn = nullptr;    // NEXT-2 seed x target matrix of the last call
    size_t conn_cap = 0;
    uint64_t last_conn_count = 0;
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
    // NEXT-4 MCMC
    cudaEvent_t mev[2] = {nullptr, nullptr};
    unsigned long long* d_mstats = nullptr;
    uint32_t* d_mvox = nullptr;     // compacted mask voxel list
    size_t mvox_cap = 0;
    uint8_t* d_mflags = nullptr;
    size_t mflags_cap = 0;
    uint8_t* d_mtemp = nullptr;     // DeviceSelect temp storage
    size_t mtemp_cap = 0;
    uint32_t* d_mcount = nullptr;   // [0] = selected voxels, [1] = work queue
    bool mcmc_done = false;
    // ablation (ii): segmented relaunch
    int32_t seg_sched[64] = {1, 2, 5, 10, 20, 50, 100, 200, 500};
    int32_t seg_n = 9;
    uint8_t* d_seg = nullptr;       // SegState arrays + second live list + select temp
    size_t seg_cap = 0;
    uint64_t m_voxels = 0, m_steps = 0;
    // last call
    bool tracked = false;
    uint64_t last_count = 0;
    uint32_t last_flags = 0;
    int32_t last_stride = 0;
    bool last_map = false;
};

static std::string g_create_err;

namespace {

pt_status fail(pt_ctx* c, pt_status s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) c->err = buf;
    else g_create_err = buf;
    return s;
}

pt_status cuda_fail(pt_ctx* c, cudaError_t e, const char* what) {
    cudaGetLastError();  // clear a non-sticky error
    if (e == cudaErrorMemoryAllocation)
        return fail(c, PT_ERR_OOM, "%s: %s", what, cudaGetErrorString(e));
    return fail(c, PT_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(expr, what)                                   \
    do {                                                 \
        cudaError_t _e = (expr);                         \
        if (_e != cudaSuccess) return cuda_fail(c, _e, what); \
    } while (0)

// RAII: make ctx's device current for the duration of a call, restore the caller's.
struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) ok = cudaSetDevice(dev) == cudaSuccess;
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

bool is_device_ptr(const void* p) {
    if (!p) return false;
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

template <typename T>
cudaError_t ensure(T*& ptr, size_t& cap, size_t n) {
    if (n <= cap && ptr) return cudaSuccess;
    if (ptr) cudaFree(ptr);
    ptr = nullptr;
    cap = 0;
    size_t want = n ? n : 1;
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(&ptr), want * sizeof(T));
    if (e == cudaSuccess) cap = want;
    return e;
}

// value of a binary16 bit pattern (exact; host side of the fp16 eligibility threshold)
static float half_bits_to_float(uint32_t h) {
    const uint32_t e = (h >> 10) & 0x1Fu, m = h & 0x3FFu;
    float v;
    if (e == 0u) v = std::ldexp((float)m, -24);
    else if (e == 31u) v = m ? NAN : INFINITY;
    else v = std::ldexp((float)(m | 0x400u), (int)e - 25);
    return (h & 0x8000u) ? -v : v;
}

int rec_bytes_of(int F, int dtype) {
    if (F < 1 || F > 3) return 0;
    int raw;
    if (dtype == PT_F32) raw = 16 * F;
    else if (dtype == PT_F16) raw = 8 * F;
    else return 0;
    return raw <= 8 ? 8 : raw <= 16 ? 16 : raw <= 32 ? 32 : 64;
}

// Device view of a caller buffer: device pointers are used in place; host inputs are
// copied into a temporary device buffer; host outputs get a temporary device buffer that
// is copied back by finish().
struct Staged {
    void* dev = nullptr;
    void* tmp = nullptr;
    void* host_out = nullptr;
    size_t bytes = 0;
    ~Staged() {
        if (tmp) cudaFree(tmp);
    }
    cudaError_t in(const void* p, size_t n, cudaStream_t st) {
        bytes = n;
        if (!p || is_device_ptr(p)) {
            dev = const_cast<void*>(p);
            return cudaSuccess;
        }
        cudaError_t e = cudaMalloc(&tmp, n ? n : 1);
        if (e != cudaSuccess) return e;
        dev = tmp;
        return cudaMemcpyAsync(tmp, p, n, cudaMemcpyHostToDevice, st);
    }
    cudaError_t out(void* p, size_t n) {
        bytes = n;
        if (!p || is_device_ptr(p)) {
            dev = p;
            return cudaSuccess;
        }
        cudaError_t e = cudaMalloc(&tmp, n ? n : 1);
        if (e != cudaSuccess) return e;
        dev = tmp;
        host_out = p;
        return cudaSuccess;
    }
    cudaError_t finish(cudaStream_t st) {
        if (!host_out) return cudaSuccess;
        return cudaMemcpyAsync(host_out, dev, bytes, cudaMemcpyDeviceToHost, st);
    }
};

}  // namespace

extern "C" {

int32_t pt_record_bytes(int32_t nfibres, int32_t dtype) { return rec_bytes_of(nfibres, dtype); }

pt_status pt_create(int cuda_device, pt_ctx** out) {
    if (!out) return fail(nullptr, PT_ERR_ARG, "pt_create: out is NULL");
    *out = nullptr;
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(nullptr, PT_ERR_CUDA, "pt_create: no CUDA device (%s)", cudaGetErrorString(e));
    }
    if (cuda_device < 0 || cuda_device >= n)
        return fail(nullptr, PT_ERR_ARG, "pt_create: device %d out of range [0,%d)", cuda_device, n);
    pt_ctx* c = new (std::nothrow) pt_ctx();
    if (!c) return fail(nullptr, PT_ERR_OOM, "pt_create: host allocation failed");
    c->device = cuda_device;
    DeviceGuard g(cuda_device);
    if (!g.ok) {
        delete c;
        return fail(nullptr, PT_ERR_CUDA, "pt_create: cudaSetDevice(%d) failed", cuda_device);
    }
    cudaDeviceProp prop;
    e = cudaGetDeviceProperties(&prop, cuda_device);
    if (e != cudaSuccess) {
        delete c;
        cudaGetLastError();
        return fail(nullptr, PT_ERR_CUDA, "pt_create: %s", cudaGetErrorString(e));
    }
    c->num_sms = prop.multiProcessorCount;
    for (auto& ev : c->mev) {
        if (cudaEventCreate(&ev) != cudaSuccess) {
            cudaGetLastError();
            pt_destroy(c);
            return fail(nullptr, PT_ERR_CUDA, "pt_create: cudaEventCreate failed");
        }
    }
    for (auto& ev : c->lev) {
        if (cudaEventCreate(&ev) != cudaSuccess) {
            cudaGetLastError();
            pt_destroy(c);
            return fail(nullptr, PT_ERR_CUDA, "pt_create: cudaEventCreate failed");
        }
    }
    for (auto& ev : c->ev) {
        if (cudaEventCreate(&ev) != cudaSuccess) {
            cudaGetLastError();
            pt_destroy(c);
            return fail(nullptr, PT_ERR_CUDA, "pt_create: cudaEventCreate failed");
        }
    }
    if (cudaMalloc(&c->d_stats, sizeof(unsigned long long) * pt::kNumStats) != cudaSuccess) {
        cudaGetLastError();
        pt_destroy(c);
        return fail(nullptr, PT_ERR_OOM, "pt_create: cudaMalloc(stats) failed");
    }
    cudaMemset(c->d_stats, 0, sizeof(unsigned long long) * pt::kNumStats);
    *out = c;
    return PT_OK;
}

void pt_destroy(pt_ctx* c) {
    if (!c) return;
    DeviceGuard g(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
    else cudaDeviceSynchronize();
    void* bufs[] = {c->d_rec, c->d_mask, c->d_seeds, c->d_ids, c->d_order, c->d_temp, c->d_map, c->d_pmap, c->d_utab,
                    c->d_stage, c->d_labels, c->d_conn, c->d_nsteps, c->d_reason, c->d_end, c->d_paths,
                    c->d_stats, c->d_mstats, c->d_mvox, c->d_mflags, c->d_mtemp, c->d_mcount, c->d_seg};
    for (void* b : bufs)
        if (b) cudaFree(b);
    for (auto& ev : c->ev)
        if (ev) cudaEventDestroy(ev);
    for (auto& ev : c->mev)
        if (ev) cudaEventDestroy(ev);
    for (auto& ev : c->lev)
        if (ev) cudaEventDestroy(ev);
    cudaGetLastError();
    delete c;
}

const char* pt_last_error(const pt_ctx* c) { return c ? c->err.c_str() : g_create_err.c_str(); }

pt_status pt_set_stream(pt_ctx* c, void* stream) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    c->stream = static_cast<cudaStream_t>(stream);
    return PT_OK;
}

pt_status pt_load_samples(pt_ctx* c, const pt_volume* v, const void* dyads, const void* f,
                          const uint8_t* mask) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!v || !dyads || !f || !mask) return fail(c, PT_ERR_ARG, "pt_load_samples: NULL argument");
    if (v->nx <= 0 || v->ny <= 0 || v->nz <= 0)
        return fail(c, PT_ERR_ARG, "pt_load_samples: dims must be > 0 (got %d %d %d)", v->nx, v->ny, v->nz);
    if (v->nsamples < 1) return fail(c, PT_ERR_ARG, "pt_load_samples: nsamples must be >= 1");
    if (v->nfibres < 1 || v->nfibres > 3)
        return fail(c, PT_ERR_ARG, "pt_load_samples: nfibres must be in [1,3] (got %d)", v->nfibres);
    const int rb = rec_bytes_of(v->nfibres, v->dtype);
    if (!rb) return fail(c, PT_ERR_ARG, "pt_load_samples: dtype must be PT_F32 or PT_F16");
    const uint64_t V = (uint64_t)v->nx * v->ny * v->nz;
    if (V > 0xFFFFFFFFull) return fail(c, PT_ERR_ARG, "pt_load_samples: more than 2^32-1 voxels");
    DeviceGuard g(c->device);
    if (!g.ok) return fail(c, PT_ERR_CUDA, "pt_load_samples: cannot select device %d", c->device);
    const uint64_t S = (uint64_t)v->nsamples, F = (uint64_t)v->nfibres;
    const size_t esz = v->dtype == PT_F16 ? 2 : 4;
    const size_t dy_bytes = F * S * V * 3 * esz, f_bytes = F * S * V * esz, m_bytes = V;
    // record layout: bricks of 2^b voxels per axis (PT_BRICK env var = b, 0 = raster)
    uint32_t blog = PT_BRICK_DEFAULT;
    if (const char* e = getenv("PT_BRICK")) blog = (uint32_t)atoi(e);
    if (blog != 0u && blog != pt::kBrickLog)
        return fail(c, PT_ERR_ARG, "pt_load_samples: PT_BRICK must be 0 (raster) or %u (16^3 bricks), got %u",
                    pt::kBrickLog, blog);
    // margin bricks (no per-step bounds test) only for volumes that stay "small"; a large
    // volume (c5) keeps the unpadded bricks, whose extra map and record footprint would cost
    const uint64_t payload = (uint64_t)V * (uint64_t)S * (uint64_t)rb;
    const pt::RecLayout L = pt::rec_layout(v->nx, v->ny, v->nz, blog, payload <= PT_BIG_VOLUME);
    if (L.nvox() > 0xFFFFFFFFull) return fail(c, PT_ERR_ARG, "pt_load_samples: padded volume exceeds 2^32-1 voxels");
    const size_t rec_size = L.nvox() * S * (size_t)rb;

    // stage host inputs on the device through one context-owned buffer (grow-only; device
    // inputs are read in place): one cudaMemcpyAsync per host array, at full speed when the
    // caller's memory is pinned
    const void* src[3] = {dyads, f, mask};
    const size_t sz[3] = {dy_bytes, f_bytes, m_bytes};
    size_t off[3], need = 0;
    bool host[3];
    for (int i = 0; i < 3; ++i) {
        host[i] = !is_device_ptr(src[i]);
        off[i] = need;
        if (host[i]) need += (sz[i] + 255) / 256 * 256;
    }
    if (need > c->stage_cap) {
        cudaStreamSynchronize(c->stream);
        if (c->d_stage) cudaFree(c->d_stage);
        c->d_stage = nullptr;
        c->stage_cap = 0;
        cudaError_t e = cudaMalloc(&c->d_stage, need);
        if (e != cudaSuccess) return cuda_fail(c, e, "pt_load_samples: staging allocation");
        c->stage_cap = need;
    }
    CK(cudaEventRecord(c->lev[0], c->stream), "pt_load_samples: event");
    const void* dsrc[3];
    c->load_h2d_bytes = 0;
    for (int i = 0; i < 3; ++i) {
        dsrc[i] = src[i];
        if (host[i]) {
            CK(cudaMemcpyAsync(c->d_stage + off[i], src[i], sz[i], cudaMemcpyHostToDevice, c->stream),
               "pt_load_samples: host-to-device copy");
            dsrc[i] = c->d_stage + off[i];
            c->load_h2d_bytes += sz[i];
        }
    }
    CK(cudaEventRecord(c->lev[1], c->stream), "pt_load_samples: event");
    const void* d_dy = dsrc[0];
    const void* d_f = dsrc[1];
    const uint8_t* d_m = static_cast<const uint8_t*>(dsrc[2]);
    if (c->d_rec && c->rec_size != rec_size) {
        cudaStreamSynchronize(c->stream);
        cudaFree(c->d_rec);
        c->d_rec = nullptr;
        c->rec_size = 0;
    }
    if (!c->d_rec) {
        cudaError_t e = cudaMalloc(&c->d_rec, rec_size);
        if (e != cudaSuccess) {
            c->loaded = false;
            return cuda_fail(c, e, "pt_load_samples: record volume allocation");
        }
        c->rec_size = rec_size;
    }
    c->loaded = false;
    cudaError_t e = ensure(c->d_mask, c->mask_cap, (size_t)V);
    if (e == cudaSuccess) e = cudaMemcpyAsync(c->d_mask, d_m, (size_t)V, cudaMemcpyDeviceToDevice, c->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(c->d_stats + pt::kStatBadInput, 0, sizeof(unsigned long long), c->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(c->d_stats + pt::kStatMaxAbs, 0, sizeof(unsigned long long), c->stream);
    if (e == cudaSuccess)
        e = pt::launch_repack(d_dy, d_f, d_m, c->d_rec, v->nx, v->ny, v->nz, L, v->nsamples, v->nfibres,
                              v->dtype == PT_F16, rb, c->d_stats + pt::kStatBadInput, c->d_stats + pt::kStatMaxAbs,
                              c->stream);
    if (e == cudaSuccess) e = cudaEventRecord(c->lev[2], c->stream);
    unsigned long long bad = 0, maxabs = 0;
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(&bad, c->d_stats + pt::kStatBadInput, sizeof bad, cudaMemcpyDeviceToHost, c->stream);
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(&maxabs, c->d_stats + pt::kStatMaxAbs, sizeof maxabs, cudaMemcpyDeviceToHost, c->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
    if (e != cudaSuccess) return cuda_fail(c, e, "pt_load_samples: repack");
    if (bad) return fail(c, PT_ERR_ARG, "pt_load_samples: %llu records inside the mask hold non-finite values", bad);
    c->vol = *v;
    c->rec_bytes = rb;
    c->layout = L;
    c->rec_payload = payload;
    {
        const uint32_t mb = (uint32_t)maxabs;
        float m;
        std::memcpy(&m, &mb, sizeof m);
        c->max_abs = m;
    }
    c->loaded = true;
    c->tracked = false;
    c->ntargets = 0;  // targets belong to a volume shape
    return PT_OK;
}

pt_status pt_track(pt_ctx* c, const float* seeds_xyz, const uint64_t* seed_ids, int64_t nseeds,
                   const pt_params* p, uint32_t* map) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!c->loaded) return fail(c, PT_ERR_STATE, "pt_track: no sample volume loaded");
    if (!p) return fail(c, PT_ERR_ARG, "pt_track: params is NULL");
    if (nseeds < 0) return fail(c, PT_ERR_ARG, "pt_track: nseeds < 0");
    if (nseeds > 0 && !seeds_xyz) return fail(c, PT_ERR_ARG, "pt_track: seeds_xyz is NULL");
    if (!(p->step > 0.f) || !std::isfinite(p->step)) return fail(c, PT_ERR_ARG, "pt_track: step must be finite and > 0");
    if (!(std::fabs(p->curv_thr) <= 1.f)) return fail(c, PT_ERR_ARG, "pt_track: |curv_thr| must be <= 1");
    if (std::isnan(p->fib_thr)) return fail(c, PT_ERR_ARG, "pt_track: fib_thr is NaN");
    if (p->max_steps < 1 || p->max_steps > 65535)
        return fail(c, PT_ERR_ARG, "pt_track: max_steps must be in [1, 65535] (got %d)", p->max_steps);
    if (p->particles_per_seed < 1) return fail(c, PT_ERR_ARG, "pt_track: particles_per_seed must be >= 1");
    if ((p->flags & PT_REC_PATHS) && p->path_stride < 1)
        return fail(c, PT_ERR_ARG, "pt_track: PT_REC_PATHS needs path_stride >= 1");
    const uint64_t P = (uint64_t)p->particles_per_seed;
    if (P > 0xFFFFFFFFull) return fail(c, PT_ERR_ARG, "pt_track: particles_per_seed must be < 2^32");
    const uint64_t N = (uint64_t)nseeds;
    if (N > 0xFFFFFFFFull) return fail(c, PT_ERR_ARG, "pt_track: more than 2^32-1 seeds");
    if (N && P > UINT64_MAX / N) return fail(c, PT_ERR_ARG, "pt_track: nseeds * P overflows");
    const uint64_t npart = N * P;
    const uint32_t fl = p->flags;
    const uint32_t kVariantFlags = PT_BIDIR | PT_INTERP | PT_INIT_RANDOM | PT_INIT_FWEIGHT | PT_KERNEL_VARIANT;
    const bool variant = (fl & kVariantFlags) != 0;
    const bool segmented = (fl & PT_KERNEL_SEGMENTED) != 0;
    const bool simple = (fl & PT_KERNEL_SIMPLE) != 0;
    const bool unique = (fl & PT_MAP_UNIQUE) != 0;
    if (segmented && (variant || unique || (fl & (PT_KERNEL_SIMPLE | PT_REC_PATHS | PT_REC_CONN))))
        return fail(c, PT_ERR_ARG, "pt_track: PT_KERNEL_SEGMENTED runs the base semantics with nsteps/reason/end outputs only");
    if (simple && (variant || unique))
        return fail(c, PT_ERR_ARG, "pt_track: PT_KERNEL_SIMPLE runs the base semantics only (no NEXT-3 variants, no PT_MAP_UNIQUE)");
    if ((fl & PT_INIT_RANDOM) && (fl & PT_INIT_FWEIGHT))
        return fail(c, PT_ERR_ARG, "pt_track: PT_INIT_RANDOM and PT_INIT_FWEIGHT are exclusive");
    if (unique && (fl & PT_MAP_ACCUMULATE) == 0 && !map)
        return fail(c, PT_ERR_ARG, "pt_track: PT_MAP_UNIQUE needs a map");
    const uint64_t H = (fl & PT_BIDIR) ? 2 : 1;   // output entries per particle
    if (npart > UINT64_MAX / 2) return fail(c, PT_ERR_ARG, "pt_track: too many particles");
    const uint64_t nout = npart * H;
    DeviceGuard g(c->device);
    if (!g.ok) return fail(c, PT_ERR_CUDA, "pt_track: cannot select device %d", c->device);
    cudaStream_t st = c->stream;

    // pid overflow: seed_id * P + (P - 1) must fit in 64 bits
    const uint64_t max_id = (UINT64_MAX - (P - 1)) / P;
    // inputs: host -> device staging
    const float* d_seeds = seeds_xyz;
    const uint64_t* d_ids = seed_ids;
    if (N && !is_device_ptr(seeds_xyz)) {
        CK(ensure(c->d_seeds, c->seeds_cap, 3 * N), "pt_track: seed buffer");
        CK(cudaMemcpyAsync(c->d_seeds, seeds_xyz, 3 * N * sizeof(float), cudaMemcpyHostToDevice, st), "pt_track: seeds H2D");
        d_seeds = c->d_seeds;
    }
    if (seed_ids) {
        if (!is_device_ptr(seed_ids)) {
            for (uint64_t i = 0; i < N; ++i)
                if (seed_ids[i] > max_id) return fail(c, PT_ERR_ARG, "pt_track: seed_id %llu * P overflows 64 bits", (unsigned long long)seed_ids[i]);
            if (N) {
                CK(ensure(c->d_ids, c->ids_cap, N), "pt_track: id buffer");
                CK(cudaMemcpyAsync(c->d_ids, seed_ids, N * sizeof(uint64_t), cudaMemcpyHostToDevice, st), "pt_track: ids H2D");
                d_ids = c->d_ids;
            }
        }
        // device-resident ids are checked by the kernel (kStatBadId -> PT_ERR_ARG in pt_get_stats)
    } else if (N && N - 1 > max_id) {
        return fail(c, PT_ERR_ARG, "pt_track: pid overflow");
    }

    const int32_t nxv = c->vol.nx, nyv = c->vol.ny, nzv = c->vol.nz;
    const uint64_t V = (uint64_t)nxv * nyv * nzv;
    const bool host_map = map && !is_device_ptr(map);
    uint32_t* d_map = map;
    if (host_map) {
        CK(ensure(c->d_map, c->map_cap, V), "pt_track: map buffer");
        d_map = c->d_map;
    }
    const bool acc = (fl & PT_MAP_ACCUMULATE) != 0;

    // outputs
    if (fl & PT_REC_LEN) CK(ensure(c->d_nsteps, c->nsteps_cap, nout), "pt_track: nsteps buffer");
    if (fl & PT_REC_REASON) CK(ensure(c->d_reason, c->reason_cap, nout), "pt_track: reason buffer");
    if (fl & PT_REC_END) CK(ensure(c->d_end, c->end_cap, 3 * nout), "pt_track: end buffer");
    if (fl & PT_REC_PATHS) {
        CK(ensure(c->d_paths, c->paths_cap, 3 * nout * (uint64_t)p->path_stride), "pt_track: path buffer");
        CK(cudaMemsetAsync(c->d_paths, 0xFF, 3 * nout * (uint64_t)p->path_stride * sizeof(float), st), "pt_track: path fill");
    }

    CK(cudaEventRecord(c->ev[0], st), "pt_track: event");
    CK(cudaMemsetAsync(c->d_stats, 0, sizeof(unsigned long long) * pt::kNumStats, st), "pt_track: stats reset");
    if (d_map) {
        if (host_map && acc)
            CK(cudaMemcpyAsync(d_map, map, V * sizeof(uint32_t), cudaMemcpyHostToDevice, st), "pt_track: map H2D");
        if (!acc) CK(cudaMemsetAsync(d_map, 0, V * sizeof(uint32_t), st), "pt_track: map zero");
        else CK(pt::launch_map_sum(d_map, (int64_t)V, c->d_stats + pt::kStatMapBefore, st), "pt_track: map sum");
    }

    // Z-order (Morton) processing order of the seeds (cub's item count is an int: above
    // INT_MAX seeds the input order is kept; results are identical either way)
    const uint32_t* d_order = nullptr;
    if (!(fl & (PT_SEED_ORDER_INPUT | PT_KERNEL_SIMPLE)) && N > 1 && N <= 0x7FFFFFFFull) {
        CK(ensure(c->d_order, c->order_cap, 4 * N), "pt_track: order buffers");
        const size_t tb = pt::seed_order_temp_bytes(N);
        CK(ensure(c->d_temp, c->temp_cap, tb), "pt_track: sort temp storage");
        CK(pt::launch_seed_order(d_seeds, N, c->d_order, c->d_order + N, c->d_order + 2 * N, c->d_order + 3 * N,
                                 c->d_temp, c->temp_cap, st),
           "pt_track: seed order");
        d_order = c->d_order + 3 * N;
    }

    const bool want_conn = (fl & PT_REC_CONN) != 0;
    if (want_conn && (c->ntargets <= 0 || !c->d_labels))
        return fail(c, PT_ERR_STATE, "pt_track: PT_REC_CONN needs targets (pt_load_targets)");
    if (want_conn) {
        CK(ensure(c->d_conn, c->conn_cap, N * (uint64_t)c->ntargets), "pt_track: connectivity buffer");
        if (N) CK(cudaMemsetAsync(c->d_conn, 0, N * (uint64_t)c->ntargets * sizeof(uint32_t), st), "pt_track: connectivity zero");
    }

    pt::TrackArgs a{};
    a.rec = c->d_rec;
    a.rb_log = c->layout.b;
    a.rb_nbx = c->layout.nbx;
    a.rb_nby = c->layout.nby;
    a.rb_off = c->layout.off;
    {
        const uint32_t b = c->layout.b, B3 = 1u << (3u * b);
        a.rb_ky = c->layout.nbx * B3 - (1u << (2u * b));
        a.rb_kz = c->layout.nbx * c->layout.nby * B3 - B3;
    }
    a.nx = nxv;
    a.ny = nyv;
    a.nz = nzv;
    a.cx = nxv / 2;
    a.cy = nyv / 2;
    a.cz = nzv / 2;
    a.fcx = (float)a.cx;
    a.fcy = (float)a.cy;
    a.fcz = (float)a.cz;
    a.pcx = a.cx + (int)c->layout.off;
    a.pcy = a.cy + (int)c->layout.off;
    a.pcz = a.cz + (int)c->layout.off;
    // every candidate stays within the margin: |step * v_a| < off - 1 voxels per axis
    a.nobounds = (c->layout.off > 0u && std::isfinite(c->max_abs) &&
                  (double)p->step * (double)c->max_abs < (double)c->layout.off - 1.0) ? 1u : 0u;
    a.S = (uint32_t)c->vol.nsamples;
    a.sample_mode = (fl & PT_SAMPLE_PER_STREAMLINE) ? 1u : 0u;
    a.step = p->step;
    a.curv_thr = p->curv_thr;
    a.fib_thr = p->fib_thr;
    a.max_steps = p->max_steps;
    a.key0 = (uint32_t)p->rng_seed;
    a.key1 = (uint32_t)(p->rng_seed >> 32);
    a.P = P;
    a.seeds = d_seeds;
    a.seed_ids = d_ids;
    a.max_seed_id = max_id;
    a.order = d_order;
    a.nseeds = N;
    a.nparticles = npart;
    {
        // a whole seed per CTA claim when there are >= 8 claims per SM, else smaller chunks
        const uint64_t P32 = (P + pt::kSub - 1) / pt::kSub * pt::kSub;
        uint64_t ch = npart / (8ull * (uint64_t)(c->num_sms > 0 ? c->num_sms : 1));
        ch = (ch + pt::kSub - 1) / pt::kSub * pt::kSub;
        if (ch < pt::kMinCtaChunk) ch = pt::kMinCtaChunk;
        if (ch > P32) ch = P32;
        if (const char* e = getenv("PT_CTA_CHUNK")) {  // experiments: particles per CTA claim
            const uint64_t v = (uint64_t)atoll(e);
            if (v >= pt::kSub) ch = (v + pt::kSub - 1) / pt::kSub * pt::kSub;
        }
        if (ch > P32) ch = P32;
        if (ch > (1ull << 27)) ch = 1ull << 27;  // keeps tickets per chunk < 2^22 (cta_take)
        a.cta_chunk = (uint32_t)ch;
    }
    a.chunks_per_seed = (uint32_t)((P + a.cta_chunk - 1) / a.cta_chunk);
    a.total_chunks = N * (uint64_t)a.chunks_per_seed;
    a.seeds_per_claim = 1;
    uint64_t spc = c->rec_payload > PT_SMALL_VOLUME ? PT_SEEDS_PER_CLAIM_BIG : PT_SEEDS_PER_CLAIM;
    if (const char* e = getenv("PT_SEEDS_PER_CLAIM")) spc = (uint64_t)atoll(e);  // experiments
    if (a.chunks_per_seed == 1 && spc > 1) {
        // whole seeds per claim: G consecutive seeds (tickets per claim must stay < 2^22)
        uint64_t G = spc;
        const uint64_t sps = (P + pt::kSub - 1) / pt::kSub;
        while (G > 1 && (G * sps >= (1ull << 22) || N / G < 8ull * (uint64_t)c->num_sms)) G >>= 1;
        // the last PT_TAIL_SEEDS_PER_SM x SMs seeds are claimed one by one (guided tail)
        const uint64_t tail = (uint64_t)PT_TAIL_SEEDS_PER_SM * (uint64_t)(c->num_sms > 0 ? c->num_sms : 1);
        a.seeds_per_claim = (uint32_t)G;
        a.group_chunks = N > tail ? (N - tail) / G : 0;
        a.total_chunks = a.group_chunks + (N - a.group_chunks * G);
    }
    a.map = d_map;
    {   // smallest binary16 pattern whose value exceeds fib_thr (fp16 records, fib_thr >= 0;
        // the finite non-negative patterns 0 .. 0x7BFF are ordered like their values)
        uint32_t lo = 0u, hi = 0x7C00u;  // 0x7C00 (+inf): no finite f is eligible
        if (p->fib_thr >= 0.f) {
            while (lo < hi) {
                const uint32_t mid = (lo + hi) / 2u;
                if (half_bits_to_float(mid) > p->fib_thr) hi = mid;
                else lo = mid + 1u;
            }
        }
        a.fib_h = (int32_t)(hi << 16);
    }
    a.o_nsteps = (fl & PT_REC_LEN) ? c->d_nsteps : nullptr;
    a.o_reason = (fl & PT_REC_REASON) ? c->d_reason : nullptr;
    a.o_end = (fl & PT_REC_END) ? c->d_end : nullptr;
    a.o_paths = (fl & PT_REC_PATHS) ? c->d_paths : nullptr;
    a.path_stride = (fl & PT_REC_PATHS) ? p->path_stride : 0;
    a.stats = c->d_stats;
    a.labels = want_conn ? c->d_labels : nullptr;
    a.ntargets = want_conn ? (uint32_t)c->ntargets : 0u;
    a.conn = want_conn ? c->d_conn : nullptr;
    a.bidir = (fl & PT_BIDIR) ? 1u : 0u;
    a.interp = (fl & PT_INTERP) ? 1u : 0u;
    a.init_mode = (fl & PT_INIT_RANDOM) ? 1u : ((fl & PT_INIT_FWEIGHT) ? 2u : 0u);
    a.mask = c->d_mask;
    a.rec_n = c->layout.nvox() * (uint64_t)c->vol.nsamples;
    a.V = V;
    a.out_n = nout;
#if PT_CHECK_BOUNDS
    // negative control of the bounds-checked build: pretend the map / mask / record buffers
    // are half their size, so in-range accesses to the upper half must be reported
    if (getenv("PT_CHECK_BOUNDS_SHRINK")) {
        a.V /= 2;
        a.rec_n /= 2;
    }
#endif
    pt::TrackMode mode;
    mode.simple = simple;
    mode.out = a.o_nsteps || a.o_reason || a.o_end || a.o_paths || a.conn;
    mode.var = variant;
    mode.unique = unique;
    if (unique && npart) {
        // one hash set per resident lane, >= 2x the most voxels a streamline can enter
        // (H halves x max_steps committed steps); the buffer is capped (PT_UNIQUE_MB, default
        // 8192 MB) by launching fewer persistent CTAs
        uint32_t ulog = 1;
        while ((1ull << ulog) < 2ull * H * (uint64_t)p->max_steps + 2ull) ++ulog;
        const uint64_t per_cta = (uint64_t)pt::kThreadsExt << ulog;  // entries (UNQ CTAs are kThreadsExt wide)
        uint64_t budget = 8192ull << 20;
        if (const char* e = getenv("PT_UNIQUE_MB")) budget = (uint64_t)atoll(e) << 20;
        uint64_t ctas = budget / (per_cta * sizeof(unsigned long long));
        if (ctas < 1) ctas = 1;
        const uint64_t full = (uint64_t)(c->num_sms > 0 ? c->num_sms : 1);
        if (ctas > full) ctas = full;
        const uint64_t need = (npart + pt::kThreadsExt - 1) / pt::kThreadsExt;
        if (ctas > need) ctas = need;
        CK(ensure(c->d_utab, c->utab_cap, (size_t)(ctas * per_cta)), "pt_track: unique-map hash sets");
        CK(cudaMemsetAsync(c->d_utab, 0, (size_t)(ctas * per_cta) * sizeof(unsigned long long), st),
           "pt_track: unique-map hash sets zero");
        a.utab = c->d_utab;
        a.ulog = ulog;
        a.max_ctas = ctas;
        a.utab_lanes = (uint32_t)(ctas * (uint64_t)pt::kThreadsExt);
    }

    // The kernels count into a context-owned scratch map, added into the caller's raster map
    // after the kernel (map_unpermute_kernel), when (a) the map is permuted -- cell of key k =
    // map_perm(k): the RED bursts of the compact neighbourhood the CTAs work on spread over
    // all L2 slices; used unless the record volume is large (c5: its records thrash L2 and
    // the map's line locality matters more) -- or (b) the launch keys the map by record voxel
    // (track_rv_keys: the bench instantiations, which then need no raster index per step).
    const bool rvk = !segmented && pt::track_rv_keys(a, mode, c->vol.dtype == PT_F16);
    a.map_keys = rvk ? c->layout.nvox() : V;
    int perm = PT_MAP_PERM;
    if (const char* e = getenv("PT_MAP_PERM")) perm = atoi(e);  // experiments
    const bool permuted = d_map && (perm == 2 || (perm == 1 && c->rec_payload <= PT_BIG_VOLUME));
    const bool scratch = d_map && (permuted || rvk);
    uint32_t pmask = 0u;
    if (scratch) {
        uint64_t cells = a.map_keys;
        if (permuted) {
            cells = 1ull << PT_MAP_GRAN;
            while (cells < a.map_keys) cells <<= 1;
            pmask = (uint32_t)((cells >> PT_MAP_GRAN) - 1);
        }
        CK(ensure(c->d_pmap, c->pmap_cap, cells), "pt_track: scratch map");
        CK(cudaMemsetAsync(c->d_pmap, 0, cells * sizeof(uint32_t), st), "pt_track: scratch map zero");
        a.map = c->d_pmap;
    }
    a.map_mask = pmask;
    // the no-bounds instantiation also takes the permuted map as given (pt_track.cuh, NOB)
    if (!permuted) a.nobounds = 0u;
    // experiment (env PT_MAP_PERSIST=1): the map as a persisting L2 access-policy window
    const bool persist = d_map && getenv("PT_MAP_PERSIST") && atoi(getenv("PT_MAP_PERSIST")) > 0;
    if (persist) {
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)V * sizeof(uint32_t));
        cudaStreamAttrValue av{};
        av.accessPolicyWindow.base_ptr = d_map;
        av.accessPolicyWindow.num_bytes = (size_t)V * sizeof(uint32_t);
        av.accessPolicyWindow.hitRatio = 1.0f;
        av.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        av.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &av);
        cudaGetLastError();
    }
    CK(cudaEventRecord(c->ev[1], st), "pt_track: event");
    if (segmented) {
        const uint32_t batch = (uint32_t)(npart < (1ull << 26) ? (npart ? npart : 1) : (1ull << 26));
        const size_t tb = pt::seg_select_temp_bytes(batch);
        const size_t per = 12 + 12 + 4 + 4 + 8 + 8 + 4 + 1 + 4;  // q p n vox pid li live flag live_b
        CK(ensure(c->d_seg, c->seg_cap, (size_t)batch * per + tb + 256 + 64), "pt_track: segment state");
        uint8_t* b = c->d_seg;
        auto take = [&](size_t bytes) {
            uint8_t* r = b;
            b += (bytes + 15) / 16 * 16;
            return r;
        };
        pt::SegState ss;
        ss.q = reinterpret_cast<float*>(take((size_t)batch * 12));
        ss.p = reinterpret_cast<float*>(take((size_t)batch * 12));
        ss.pid = reinterpret_cast<uint64_t*>(take((size_t)batch * 8));
        ss.li = reinterpret_cast<uint64_t*>(take((size_t)batch * 8));
        ss.n = reinterpret_cast<uint32_t*>(take((size_t)batch * 4));
        ss.vox = reinterpret_cast<uint32_t*>(take((size_t)batch * 4));
        ss.live = reinterpret_cast<uint32_t*>(take((size_t)batch * 4));
        uint32_t* live_b = reinterpret_cast<uint32_t*>(take((size_t)batch * 4));
        uint32_t* d_count = reinterpret_cast<uint32_t*>(take(16));
        ss.flag = take((size_t)batch);
        void* temp = take(tb);
        CK(pt::run_segmented(a, c->vol.nfibres, c->vol.dtype == PT_F16, ss, batch, c->seg_sched, c->seg_n, live_b,
                             d_count, temp, tb, st),
           "pt_track: segmented relaunch");
    } else {
        CK(pt::launch_track(a, mode, c->vol.nfibres, c->vol.dtype == PT_F16, c->num_sms, st),
           "pt_track: tracking kernel launch");
    }
    CK(cudaEventRecord(c->ev[2], st), "pt_track: event");
    if (persist) {
        cudaStreamAttrValue av{};
        av.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &av);
        cudaCtxResetPersistingL2Cache();
        cudaGetLastError();
    }
    if (scratch)
        CK(pt::launch_map_unpermute(c->d_pmap, pmask, rvk, nxv, nyv, c->layout, d_map, (int64_t)V, true, st),
           "pt_track: scratch map add");
    if (d_map) CK(pt::launch_map_sum(d_map, (int64_t)V, c->d_stats + pt::kStatMapAfter, st), "pt_track: map sum");
    if (host_map) {
        CK(cudaMemcpyAsync(map, d_map, V * sizeof(uint32_t), cudaMemcpyDeviceToHost, st), "pt_track: map D2H");
    }
    CK(cudaEventRecord(c->ev[3], st), "pt_track: event");
    if (host_map) CK(cudaStreamSynchronize(st), "pt_track: synchronise");

    c->tracked = true;
    c->last_count = nout;
    c->last_flags = fl;
    c->last_stride = (fl & PT_REC_PATHS) ? p->path_stride : 0;
    c->last_map = d_map != nullptr;
    c->last_conn_count = want_conn ? N * (uint64_t)c->ntargets : 0;
    return PT_OK;
}

pt_status pt_set_segments(pt_ctx* c, const int32_t* intervals, int32_t n) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!intervals || n < 1 || n > 64) return fail(c, PT_ERR_ARG, "pt_set_segments: need 1..64 intervals");
    for (int32_t i = 0; i < n; ++i)
        if (intervals[i] < 1) return fail(c, PT_ERR_ARG, "pt_set_segments: interval %d < 1", i);
    for (int32_t i = 0; i < n; ++i) c->seg_sched[i] = intervals[i];
    c->seg_n = n;
    return PT_OK;
}

pt_status pt_load_targets(pt_ctx* c, const uint8_t* labels, int32_t ntargets) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!c->loaded) return fail(c, PT_ERR_STATE, "pt_load_targets: load the sample volume first");
    if (ntargets < 0 || ntargets > 64) return fail(c, PT_ERR_ARG, "pt_load_targets: ntargets must be in [0, 64]");
    if (!labels || ntargets == 0) {
        c->ntargets = 0;
        return PT_OK;
    }
    DeviceGuard g(c->device);
    const size_t V = (size_t)c->vol.nx * c->vol.ny * c->vol.nz;
    CK(ensure(c->d_labels, c->labels_cap, V), "pt_load_targets: label buffer");
    CK(cudaMemcpyAsync(c->d_labels, labels, V, cudaMemcpyDefault, c->stream), "pt_load_targets: copy");
    c->ntargets = 0;
    CK(cudaMemsetAsync(c->d_stats + pt::kStatLabelMax, 0, sizeof(unsigned long long), c->stream), "pt_load_targets: reset");
    CK(pt::launch_label_max(c->d_labels, (int64_t)V, c->d_stats + pt::kStatLabelMax, c->stream), "pt_load_targets: scan");
    unsigned long long lmax = 0;
    CK(cudaMemcpyAsync(&lmax, c->d_stats + pt::kStatLabelMax, sizeof lmax, cudaMemcpyDeviceToHost, c->stream),
       "pt_load_targets: scan result");
    CK(cudaStreamSynchronize(c->stream), "pt_load_targets: synchronise");
    if (lmax > (unsigned long long)ntargets)
        return fail(c, PT_ERR_ARG, "pt_load_targets: label %llu > ntargets %d", lmax, ntargets);
    c->ntargets = ntargets;
    return PT_OK;
}

pt_status pt_get_connectivity(pt_ctx* c, uint32_t* out, int64_t capacity, int64_t* count) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!c->tracked || c->last_conn_count == 0)
        return fail(c, PT_ERR_STATE, "pt_get_connectivity: the last pt_track did not record PT_REC_CONN");
    if (count) *count = (int64_t)c->last_conn_count;
    if (!out) return PT_OK;
    if (capacity < (int64_t)c->last_conn_count)
        return fail(c, PT_ERR_ARG, "pt_get_connectivity: capacity %lld < %llu", (long long)capacity,
                    (unsigned long long)c->last_conn_count);
    DeviceGuard g(c->device);
    CK(cudaMemcpyAsync(out, c->d_conn, c->last_conn_count * sizeof(uint32_t), cudaMemcpyDefault, c->stream),
       "pt_get_connectivity: copy");
    CK(cudaStreamSynchronize(c->stream), "pt_get_connectivity: synchronise");
    return PT_OK;
}

pt_status pt_get_stats(pt_ctx* c, pt_stats* out) {
    if (!c || !out) return PT_ERR_ARG;
    c->err.clear();
    if (!c->tracked) return fail(c, PT_ERR_STATE, "pt_get_stats: no pt_track yet");
    DeviceGuard g(c->device);
    unsigned long long s[pt::kNumStats];
    CK(cudaStreamSynchronize(c->stream), "pt_get_stats: synchronise");
    CK(cudaMemcpy(s, c->d_stats, sizeof s, cudaMemcpyDeviceToHost), "pt_get_stats: copy");
    std::memset(out, 0, sizeof *out);
    out->total_steps = s[pt::kStatSteps];
    out->particles = s[pt::kStatParticles];
    out->lane_active = s[pt::kStatLaneActive];
    out->lane_slots = s[pt::kStatLaneSlots];
    out->map_sum = s[pt::kStatMapAfter];
    out->unique_visits = s[pt::kStatUnique];
    // the map gains one count per committed step (R13), or per first entry with PT_MAP_UNIQUE
    const unsigned long long added = (c->last_flags & PT_MAP_UNIQUE) ? s[pt::kStatUnique] : s[pt::kStatSteps];
    out->overflow = (c->last_map && s[pt::kStatMapAfter] != s[pt::kStatMapBefore] + added) ? 1 : 0;
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, c->ev[1], c->ev[2]), "pt_get_stats: kernel time");
    out->kernel_ms = ms;
    CK(cudaEventElapsedTime(&ms, c->ev[0], c->ev[3]), "pt_get_stats: track time");
    out->track_ms = ms;
    if (s[pt::kStatBadAccess])
        return fail(c, PT_ERR_CUDA, "bounds check (PT_CHECK_BOUNDS build): a tracking kernel accessed outside a buffer");
    if (s[pt::kStatBadId])
        return fail(c, PT_ERR_ARG, "pt_track: a device-resident seed_id * P overflows 64 bits (those particles ran as seed id 0)");
    if (out->overflow) return fail(c, PT_ERR_OVERFLOW, "a uint32 map cell wrapped past 2^32-1");
    return PT_OK;
}

pt_status pt_get_paths(pt_ctx* c, pt_paths* out) {
    if (!c || !out) return PT_ERR_ARG;
    c->err.clear();
    if (!c->tracked) return fail(c, PT_ERR_STATE, "pt_get_paths: no pt_track yet");
    DeviceGuard g(c->device);
    out->count = (int64_t)c->last_count;
    out->path_stride = c->last_stride;
    const bool any = out->nsteps || out->reason || out->end_xyz || out->paths;
    if (any && out->capacity < (int64_t)c->last_count)
        return fail(c, PT_ERR_ARG, "pt_get_paths: capacity %lld < count %llu", (long long)out->capacity,
                    (unsigned long long)c->last_count);
    if ((out->nsteps && !(c->last_flags & PT_REC_LEN)) || (out->reason && !(c->last_flags & PT_REC_REASON)) ||
        (out->end_xyz && !(c->last_flags & PT_REC_END)) || (out->paths && !(c->last_flags & PT_REC_PATHS)))
        return fail(c, PT_ERR_STATE, "pt_get_paths: output not recorded by the last pt_track (flags 0x%x)", c->last_flags);
    const uint64_t n = c->last_count;
    cudaStream_t st = c->stream;
    if (n) {
        if (out->nsteps) CK(cudaMemcpyAsync(out->nsteps, c->d_nsteps, n * 2, cudaMemcpyDefault, st), "pt_get_paths: nsteps");
        if (out->reason) CK(cudaMemcpyAsync(out->reason, c->d_reason, n, cudaMemcpyDefault, st), "pt_get_paths: reason");
        if (out->end_xyz) CK(cudaMemcpyAsync(out->end_xyz, c->d_end, n * 12, cudaMemcpyDefault, st), "pt_get_paths: end");
        if (out->paths)
            CK(cudaMemcpyAsync(out->paths, c->d_paths, n * 12 * (uint64_t)c->last_stride, cudaMemcpyDefault, st),
               "pt_get_paths: paths");
    }
    CK(cudaStreamSynchronize(st), "pt_get_paths: synchronise");
    pt_stats s;
    pt_status rc = pt_get_stats(c, &s);
    return rc;
}

pt_status pt_get_load_stats(pt_ctx* c, pt_load_stats* out) {
    if (!c || !out) return PT_ERR_ARG;
    c->err.clear();
    if (!c->loaded) return fail(c, PT_ERR_STATE, "pt_get_load_stats: no sample volume loaded");
    DeviceGuard g(c->device);
    float a = 0.f, b = 0.f;
    CK(cudaEventElapsedTime(&a, c->lev[0], c->lev[1]), "pt_get_load_stats: h2d time");
    CK(cudaEventElapsedTime(&b, c->lev[1], c->lev[2]), "pt_get_load_stats: repack time");
    out->h2d_ms = a;
    out->repack_ms = b;
    out->h2d_bytes = c->load_h2d_bytes;
    out->record_bytes = c->rec_size;
    return PT_OK;
}

pt_status pt_rng_draws(pt_ctx* c, const uint64_t* pid, const uint32_t* block, const uint32_t* stream, int64_t n,
                       uint64_t rng_seed, uint32_t nsamples, uint32_t* words, uint32_t* samples,
                       int64_t* mismatches) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (n < 0 || nsamples < 1 || (n > 0 && (!pid || !block || !stream || !words || !samples)) || !mismatches)
        return fail(c, PT_ERR_ARG, "pt_rng_draws: NULL array, n < 0 or nsamples < 1");
    DeviceGuard g(c->device);
    cudaStream_t st = c->stream;
    const size_t un = (size_t)n;
    Staged sp, sb, ss, sw, sm;
    CK(sp.in(pid, un * 8, st), "pt_rng_draws: pid");
    CK(sb.in(block, un * 4, st), "pt_rng_draws: block");
    CK(ss.in(stream, un * 4, st), "pt_rng_draws: stream");
    CK(sw.out(words, un * 16), "pt_rng_draws: words");
    CK(sm.out(samples, un * 12), "pt_rng_draws: samples");
    CK(cudaMemsetAsync(c->d_stats + pt::kStatLabelMax, 0, sizeof(unsigned long long), st), "pt_rng_draws: reset");
    CK(pt::launch_rng_draws(static_cast<const uint64_t*>(sp.dev), static_cast<const uint32_t*>(sb.dev),
                            static_cast<const uint32_t*>(ss.dev), n, (uint32_t)rng_seed, (uint32_t)(rng_seed >> 32),
                            nsamples, static_cast<uint32_t*>(sw.dev), static_cast<uint32_t*>(sm.dev),
                            c->d_stats + pt::kStatLabelMax, st),
       "pt_rng_draws: kernel");
    CK(sw.finish(st), "pt_rng_draws: words D2H");
    CK(sm.finish(st), "pt_rng_draws: samples D2H");
    unsigned long long mm = 0;
    CK(cudaMemcpyAsync(&mm, c->d_stats + pt::kStatLabelMax, sizeof mm, cudaMemcpyDeviceToHost, st), "pt_rng_draws: count");
    CK(cudaStreamSynchronize(st), "pt_rng_draws: synchronise");
    *mismatches = (int64_t)mm;
    return PT_OK;
}

pt_status pt_gather_bench(pt_ctx* c, int64_t buffer_bytes, int32_t record_bytes, double* sectors_per_s) {
    if (!c || !sectors_per_s) return PT_ERR_ARG;
    c->err.clear();
    if (record_bytes != 8 && record_bytes != 16 && record_bytes != 32 && record_bytes != 64)
        return fail(c, PT_ERR_ARG, "pt_gather_bench: record_bytes must be 8, 16, 32 or 64");
    if (buffer_bytes < record_bytes * 1024)
        return fail(c, PT_ERR_ARG, "pt_gather_bench: buffer too small");
    DeviceGuard g(c->device);
    uint8_t* buf = nullptr;
    uint32_t* sink = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    auto cleanup = [&]() {
        if (buf) cudaFree(buf);
        if (sink) cudaFree(sink);
        if (e0) cudaEventDestroy(e0);
        if (e1) cudaEventDestroy(e1);
    };
    cudaError_t e = cudaMalloc(&buf, (size_t)buffer_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&sink, 64);
    if (e == cudaSuccess) e = cudaMemsetAsync(buf, 0x3C, (size_t)buffer_bytes, c->stream);
    if (e == cudaSuccess) e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    if (e != cudaSuccess) {
        cleanup();
        return cuda_fail(c, e, "pt_gather_bench: setup");
    }
    const uint64_t nrec = (uint64_t)buffer_bytes / (uint64_t)record_bytes;
    int per_sm = pt::gather_bench_blocks_per_sm(record_bytes);
    if (per_sm < 1) per_sm = 1;
    const int blocks = c->num_sms * per_sm;
    const uint32_t iters = 256;
    double best = 0.0;
    for (int rep = 0; rep < 4; ++rep) {
        e = cudaEventRecord(e0, c->stream);
        if (e == cudaSuccess) e = pt::launch_gather_bench(buf, nrec, record_bytes, iters, blocks, 0x1234567u + rep, sink, c->stream);
        if (e == cudaSuccess) e = cudaEventRecord(e1, c->stream);
        if (e == cudaSuccess) e = cudaEventSynchronize(e1);
        float ms = 0.f;
        if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, e0, e1);
        if (e != cudaSuccess) {
            cleanup();
            return cuda_fail(c, e, "pt_gather_bench: run");
        }
        const double loads = (double)blocks * 256.0 * (double)iters;
        const double sectors = loads * (record_bytes > 32 ? record_bytes / 32 : 1);
        const double rate = sectors / (ms * 1e-3);
        if (rep > 0 && rate > best) best = rate;  // rep 0 = warm-up
    }
    cleanup();
    *sectors_per_s = best;
    return PT_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------- NEXT-4 MCMC


extern "C" {

pt_status pt_mcmc(pt_ctx* c, const pt_dwi_shape* sh, const float* dwi, const float* bvals, const float* bvecs,
                  const uint8_t* mask, const pt_mcmc_params* p, const double* init, double* samples,
                  uint32_t* accepted) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!sh || !p || !dwi || !bvals || !bvecs || !mask || !samples)
        return fail(c, PT_ERR_ARG, "pt_mcmc: NULL argument");
    if (sh->nx <= 0 || sh->ny <= 0 || sh->nz <= 0) return fail(c, PT_ERR_ARG, "pt_mcmc: dims must be > 0");
    if (sh->nmeas < 1 || sh->nmeas > 128) return fail(c, PT_ERR_ARG, "pt_mcmc: nmeas must be in [1, 128]");
    if (p->nfibres < 1 || p->nfibres > 3) return fail(c, PT_ERR_ARG, "pt_mcmc: nfibres must be in [1, 3]");
    if (p->burnin < 0 || p->nsamples < 1 || p->interval < 1 || p->adapt_every < 1)
        return fail(c, PT_ERR_ARG, "pt_mcmc: burnin >= 0, nsamples >= 1, interval >= 1, adapt_every >= 1");
    const uint64_t loops = (uint64_t)p->burnin + (uint64_t)p->nsamples * (uint64_t)p->interval;
    if (loops >= 0xFFFFFFFFull) return fail(c, PT_ERR_ARG, "pt_mcmc: burnin + nsamples * interval >= 2^32");
    const uint64_t V = (uint64_t)sh->nx * sh->ny * sh->nz;
    if (V > 0xFFFFFFFFull) return fail(c, PT_ERR_ARG, "pt_mcmc: more than 2^32-1 voxels");
    const int N = p->nfibres, NP = 3 + 3 * N;
    const uint32_t fixed = p->fixed & ((1u << NP) - 1u);
    DeviceGuard g(c->device);
    if (!g.ok) return fail(c, PT_ERR_CUDA, "pt_mcmc: cannot select device %d", c->device);
    cudaStream_t st = c->stream;
    const size_t n = (size_t)sh->nmeas;
    Staged sd, sb, sv, sm, si, ss, sa;
    CK(sd.in(dwi, n * V * sizeof(float), st), "pt_mcmc: dwi");
    CK(sb.in(bvals, n * sizeof(float), st), "pt_mcmc: bvals");
    CK(sv.in(bvecs, 3 * n * sizeof(float), st), "pt_mcmc: bvecs");
    CK(sm.in(mask, V, st), "pt_mcmc: mask");
    CK(si.in(init, init ? (size_t)NP * V * sizeof(double) : 0, st), "pt_mcmc: init");
    CK(ss.out(samples, (size_t)NP * (size_t)p->nsamples * V * sizeof(double)), "pt_mcmc: samples buffer");
    CK(sa.out(accepted, accepted ? (size_t)NP * V * sizeof(uint32_t) : 0), "pt_mcmc: accepted buffer");
    if (!c->d_mstats) CK(cudaMalloc(&c->d_mstats, sizeof(unsigned long long) * pt::kMcmcNumStats), "pt_mcmc: stats");
    if (!c->d_mcount) CK(cudaMalloc(&c->d_mcount, 2 * sizeof(uint32_t)), "pt_mcmc: counters");
    CK(ensure(c->d_mvox, c->mvox_cap, V), "pt_mcmc: voxel list");
    CK(ensure(c->d_mflags, c->mflags_cap, V), "pt_mcmc: flags");
    CK(ensure(c->d_mtemp, c->mtemp_cap, pt::mcmc_select_temp_bytes(V)), "pt_mcmc: select temp");
    CK(cudaMemsetAsync(c->d_mcount, 0, 2 * sizeof(uint32_t), st), "pt_mcmc: counters zero");
    CK(cudaMemsetAsync(c->d_mstats, 0, sizeof(unsigned long long) * pt::kMcmcNumStats, st), "pt_mcmc: stats zero");
    CK(cudaMemsetAsync(ss.dev, 0, ss.bytes, st), "pt_mcmc: samples zero");
    if (sa.dev) CK(cudaMemsetAsync(sa.dev, 0, sa.bytes, st), "pt_mcmc: accepted zero");
    CK(pt::launch_mcmc_voxel_list(static_cast<const uint8_t*>(sm.dev), V, c->d_mflags, c->d_mvox, c->d_mcount,
                                  c->d_mtemp, c->mtemp_cap, st),
       "pt_mcmc: voxel list");
    uint32_t nvox = 0;
    CK(cudaMemcpyAsync(&nvox, c->d_mcount, sizeof nvox, cudaMemcpyDeviceToHost, st), "pt_mcmc: count");
    CK(cudaStreamSynchronize(st), "pt_mcmc: synchronise");

    pt::McmcArgs a{};
    a.dwi = static_cast<const float*>(sd.dev);
    a.bvals = static_cast<const float*>(sb.dev);
    a.bvecs = static_cast<const float*>(sv.dev);
    a.vox = c->d_mvox;
    a.nvox = nvox;
    a.queue = c->d_mcount + 1;
    a.V = V;
    a.nmeas = sh->nmeas;
    a.nfibres = N;
    a.burnin = (uint32_t)p->burnin;
    a.nsamples = (uint32_t)p->nsamples;
    a.interval = (uint32_t)p->interval;
    a.adapt_every = (uint32_t)p->adapt_every;
    a.loops = (uint32_t)loops;
    a.key0 = (uint32_t)p->rng_seed;
    a.key1 = (uint32_t)(p->rng_seed >> 32);
    a.fixed = fixed;
    a.init = static_cast<const double*>(si.dev);
    a.samples = static_cast<double*>(ss.dev);
    a.accepted = static_cast<uint32_t*>(sa.dev);
    a.stats = c->d_mstats;
    CK(cudaEventRecord(c->mev[0], st), "pt_mcmc: event");
    if (nvox) CK(pt::launch_mcmc(a, c->num_sms, st), "pt_mcmc: kernel launch");
    CK(cudaEventRecord(c->mev[1], st), "pt_mcmc: event");
    CK(ss.finish(st), "pt_mcmc: samples D2H");
    CK(sa.finish(st), "pt_mcmc: accepted D2H");
    CK(cudaStreamSynchronize(st), "pt_mcmc: synchronise");
    c->mcmc_done = true;
    c->m_voxels = nvox;
    c->m_steps = (uint64_t)nvox * loops * (uint64_t)(NP - __builtin_popcount(fixed));
    return PT_OK;
}

pt_status pt_get_mcmc_stats(pt_ctx* c, pt_mcmc_stats* out) {
    if (!c || !out) return PT_ERR_ARG;
    c->err.clear();
    if (!c->mcmc_done) return fail(c, PT_ERR_STATE, "pt_get_mcmc_stats: no pt_mcmc yet");
    DeviceGuard g(c->device);
    unsigned long long s[pt::kMcmcNumStats];
    CK(cudaStreamSynchronize(c->stream), "pt_get_mcmc_stats: synchronise");
    CK(cudaMemcpy(s, c->d_mstats, sizeof s, cudaMemcpyDeviceToHost), "pt_get_mcmc_stats: copy");
    out->voxels = c->m_voxels;
    out->mh_steps = c->m_steps;
    out->accepted = s[pt::kMcmcStatAccepted];
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, c->mev[0], c->mev[1]), "pt_get_mcmc_stats: kernel time");
    out->kernel_ms = ms;
    if (s[pt::kMcmcStatBadAccess])
        return fail(c, PT_ERR_CUDA, "bounds check (PT_CHECK_BOUNDS build): the MCMC kernel accessed outside a buffer");
    return PT_OK;
}

pt_status pt_mcmc_to_volume(pt_ctx* c, const pt_dwi_shape* sh, int32_t nfibres, int32_t nsamples,
                            const double* samples, const uint8_t* mask, float* dyads, float* f) {
    if (!c) return PT_ERR_ARG;
    c->err.clear();
    if (!sh || !samples || !mask || !dyads || !f) return fail(c, PT_ERR_ARG, "pt_mcmc_to_volume: NULL argument");
    if (sh->nx <= 0 || sh->ny <= 0 || sh->nz <= 0) return fail(c, PT_ERR_ARG, "pt_mcmc_to_volume: dims must be > 0");
    if (nfibres < 1 || nfibres > 3 || nsamples < 1)
        return fail(c, PT_ERR_ARG, "pt_mcmc_to_volume: nfibres in [1, 3], nsamples >= 1");
    const uint64_t V = (uint64_t)sh->nx * sh->ny * sh->nz;
    DeviceGuard g(c->device);
    cudaStream_t st = c->stream;
    const size_t NP = 3 + 3 * (size_t)nfibres;
    Staged ss, sm, sd, sf;
    CK(ss.in(samples, NP * (size_t)nsamples * V * sizeof(double), st), "pt_mcmc_to_volume: samples");
    CK(sm.in(mask, V, st), "pt_mcmc_to_volume: mask");
    CK(sd.out(dyads, (size_t)nfibres * nsamples * V * 3 * sizeof(float)), "pt_mcmc_to_volume: dyads");
    CK(sf.out(f, (size_t)nfibres * nsamples * V * sizeof(float)), "pt_mcmc_to_volume: f");
    CK(pt::launch_samples_to_volume(static_cast<const double*>(ss.dev), static_cast<const uint8_t*>(sm.dev), V,
                                    nfibres, nsamples, static_cast<float*>(sd.dev), static_cast<float*>(sf.dev), st),
       "pt_mcmc_to_volume: kernel");
    CK(sd.finish(st), "pt_mcmc_to_volume: dyads D2H");
    CK(sf.finish(st), "pt_mcmc_to_volume: f D2H");
    CK(cudaStreamSynchronize(st), "pt_mcmc_to_volume: synchronise");
    return PT_OK;
}

}  // extern "C"
