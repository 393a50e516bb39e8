// pt_kernels.cu -- sm_100a kernels of the probabilistic-streamlining hot path besides the
// stepping kernel itself (pt_track.cuh, instantiated in pt_track_f{1,2,3}.cu):
//
//   repack_kernel  : canonical sample volumes -> one record per (voxel, sample)
//   map_sum_kernel : sum of the uint32 map (overflow detection, R17)
//   gather_bench   : random-record gather micro-benchmark (roofline denominator)
//
#include <cuda_runtime.h>
#include <cub/device/device_radix_sort.cuh>
#include <curand_philox4x32_x.h>

#include <cstdint>

#include "pt_device.cuh"
#include "pt_internal.h"

namespace pt {

// ------------------------------------------------------------------------- repack
// Canonical [F][S][Z][Y][X](x3) sample volumes -> rec[vox][s] (one thread per record,
// s fastest so the record stores are coalesced).  Voxels outside the mask get the
// sentinel f0 = all-ones; non-finite values inside the mask are counted in *bad.
template <bool HALF>
__global__ void repack_kernel(const void* __restrict__ dyads, const void* __restrict__ fr,
                              const uint8_t* __restrict__ mask, uint8_t* __restrict__ rec,
                              int nx, int ny, int64_t V, RecLayout L, int S, int F, int RB,
                              unsigned long long* bad, unsigned long long* maxabs) {
    float vmax = 0.f;  // largest |vector component| of this thread's records inside the mask
    const int64_t total = V * (int64_t)S;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t vox = i / S;
        const int s = (int)(i - vox * S);
        uint32_t w[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) w[k] = 0u;
        const bool inside = mask[vox] != 0;
        bool ok = true;
        for (int j = 0; j < F; ++j) {
            const int64_t e = ((int64_t)j * S + s) * V + vox;
            if (HALF) {
                const uint16_t* d = static_cast<const uint16_t*>(dyads);
                const uint16_t* f = static_cast<const uint16_t*>(fr);
                const uint16_t x = d[3 * e], y = d[3 * e + 1], z = d[3 * e + 2], ff = f[e];
                ok = ok && ((x & 0x7C00u) != 0x7C00u) && ((y & 0x7C00u) != 0x7C00u) &&
                     ((z & 0x7C00u) != 0x7C00u) && ((ff & 0x7C00u) != 0x7C00u);
                w[2 * j] = (uint32_t)x | ((uint32_t)y << 16);
                w[2 * j + 1] = (uint32_t)z | ((uint32_t)ff << 16);
            } else {
                const float* d = static_cast<const float*>(dyads);
                const float* f = static_cast<const float*>(fr);
                const float x = d[3 * e], y = d[3 * e + 1], z = d[3 * e + 2], ff = f[e];
                ok = ok && isfinite(x) && isfinite(y) && isfinite(z) && isfinite(ff);
                w[4 * j] = __float_as_uint(x);
                w[4 * j + 1] = __float_as_uint(y);
                w[4 * j + 2] = __float_as_uint(z);
                w[4 * j + 3] = __float_as_uint(ff);
            }
        }
        if (!inside) {
            if (HALF) w[1] |= 0xFFFF0000u;
            else w[3] = 0xFFFFFFFFu;
        } else if (!ok) {
            atomicAdd(bad, 1ull);
        } else {
            for (int j = 0; j < F; ++j) {
                float c[3];
                if (HALF) {
                    c[0] = __half2float(__ushort_as_half((unsigned short)(w[2 * j] & 0xFFFFu)));
                    c[1] = __half2float(__ushort_as_half((unsigned short)(w[2 * j] >> 16)));
                    c[2] = __half2float(__ushort_as_half((unsigned short)(w[2 * j + 1] & 0xFFFFu)));
                } else {
                    c[0] = __uint_as_float(w[4 * j]);
                    c[1] = __uint_as_float(w[4 * j + 1]);
                    c[2] = __uint_as_float(w[4 * j + 2]);
                }
                for (int k = 0; k < 3; ++k) vmax = fmaxf(vmax, fabsf(c[k]));
            }
        }
        const uint64_t rv = rec_vox_raster((uint32_t)vox, (uint32_t)nx, (uint32_t)ny, L.b, L.nbx, L.nby, L.off);
        uint8_t* out = rec + rec_slot((uint32_t)rv, (uint32_t)s, (uint32_t)S, L.b) * RB;
        if (RB == 8) {
            *reinterpret_cast<uint2*>(out) = make_uint2(w[0], w[1]);
        } else {
            for (int k = 0; k < RB / 16; ++k)
                reinterpret_cast<uint4*>(out)[k] = make_uint4(w[4 * k], w[4 * k + 1], w[4 * k + 2], w[4 * k + 3]);
        }
    }
    // non-negative floats order like their bit patterns
    const unsigned m = __reduce_max_sync(kFull, __float_as_uint(vmax));
    if ((threadIdx.x & 31u) == 0u && m) atomicMax(maxabs, (unsigned long long)m);
}

// ------------------------------------------------------------------------- seed order
// Morton key of the seed's voxel (10 bits per axis; coordinates clamped to [0, 1023]),
// with the input index in the low 32 bits so the sort is a total order.
__device__ __forceinline__ uint64_t spread3(uint32_t v) {
    uint64_t x = v & 0x3FFu;
    x = (x | (x << 16)) & 0x030000FFull;
    x = (x | (x << 8)) & 0x0300F00Full;
    x = (x | (x << 4)) & 0x030C30C3ull;
    x = (x | (x << 2)) & 0x09249249ull;
    return x;
}

__global__ void seed_keys_kernel(const float* __restrict__ seeds, uint64_t n, uint32_t* keys,
                                 uint32_t* idx) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t c[3];
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            const float x = seeds[3 * i + a];
            c[a] = x <= 0.f ? 0u : (x >= 1023.f ? 1023u : (uint32_t)x);
        }
        keys[i] = (uint32_t)(spread3(c[0]) | (spread3(c[1]) << 1) | (spread3(c[2]) << 2));
        idx[i] = (uint32_t)i;
    }
}

// (the caller keeps nseeds <= INT_MAX: cub's num_items is an int here)
size_t seed_order_temp_bytes(uint64_t nseeds) {
    size_t bytes = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, bytes, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                    (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)nseeds, 0, 30);
    return bytes;
}

cudaError_t launch_seed_order(const float* seeds, uint64_t nseeds, uint32_t* keys, uint32_t* keys_out,
                              uint32_t* idx, uint32_t* perm, void* temp, size_t temp_bytes, cudaStream_t st) {
    if (nseeds == 0) return cudaSuccess;
    uint64_t blocks = (nseeds + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    seed_keys_kernel<<<(unsigned)blocks, 256, 0, st>>>(seeds, nseeds, keys, idx);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    // stable radix sort on the 30-bit Morton code: ties keep the input order
    return cub::DeviceRadixSort::SortPairs(temp, temp_bytes, keys, keys_out, idx, perm, (int)nseeds, 0, 30, st);
}

// ------------------------------------------------------------------------- map sum
__global__ void map_sum_kernel(const uint32_t* __restrict__ map, int64_t V, unsigned long long* out) {
    unsigned long long s = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += (int64_t)gridDim.x * blockDim.x)
        s += map[i];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

__global__ void map_unpermute_kernel(const uint32_t* __restrict__ pm, uint32_t mask, bool rvk, uint32_t nx,
                                     uint32_t ny, RecLayout L, uint32_t* __restrict__ map, int64_t V, bool acc) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t key = rvk ? rec_vox_raster((uint32_t)i, nx, ny, L.b, L.nbx, L.nby, L.off) : (uint32_t)i;
        const uint32_t c = pm[mask ? map_perm(key, mask) : key];
        map[i] = acc ? map[i] + c : c;
    }
}

// ------------------------------------------------------------------------- RNG self-test
// The tracking kernel's own Philox and sample-index functions on explicit counters, with
// the CUDA library's curand_Philox4x32_10 as an independent cross-check (pt_rng_draws).
__global__ void rng_draws_kernel(const uint64_t* __restrict__ pid, const uint32_t* __restrict__ block,
                                 const uint32_t* __restrict__ stream, int64_t n, uint32_t k0, uint32_t k1,
                                 uint32_t S, uint32_t* __restrict__ words, uint32_t* __restrict__ samples,
                                 unsigned long long* mismatches) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const uint4 c = make_uint4(block[i], (uint32_t)pid[i], (uint32_t)(pid[i] >> 32), stream[i]);
        const uint4 w = philox4x32_10(c, k0, k1);
        const uint4 r = curand_Philox4x32_10(c, make_uint2(k0, k1));
        if (w.x != r.x || w.y != r.y || w.z != r.z || w.w != r.w) atomicAdd(mismatches, 1ull);
        words[4 * i + 0] = w.x;
        words[4 * i + 1] = w.y;
        words[4 * i + 2] = w.z;
        words[4 * i + 3] = w.w;
        samples[3 * i + 0] = sample_of(w.x, S);
        samples[3 * i + 1] = sample_of(w.y, S);
        samples[3 * i + 2] = sample_of(w.z, S);
    }
}

cudaError_t launch_rng_draws(const uint64_t* pid, const uint32_t* block, const uint32_t* stream, int64_t n,
                             uint32_t k0, uint32_t k1, uint32_t S, uint32_t* words, uint32_t* samples,
                             unsigned long long* mismatches, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    int64_t blocks = (n + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    rng_draws_kernel<<<(unsigned)blocks, 256, 0, st>>>(pid, block, stream, n, k0, k1, S, words, samples, mismatches);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------- label max
__global__ void label_max_kernel(const uint8_t* __restrict__ lab, int64_t V, unsigned long long* out) {
    uint32_t m = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += (int64_t)gridDim.x * blockDim.x)
        m = max(m, (uint32_t)lab[i]);
    m = __reduce_max_sync(kFull, m);
    if ((threadIdx.x & 31) == 0 && m) atomicMax(out, (unsigned long long)m);
}

cudaError_t launch_label_max(const uint8_t* labels, int64_t V, unsigned long long* out, cudaStream_t st) {
    int64_t blocks = (V + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    label_max_kernel<<<(unsigned)blocks, 256, 0, st>>>(labels, V, out);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------- gather bench
// Uniformly random record-aligned reads, 8 independent loads in flight per thread.
template <int RB>
__global__ void __launch_bounds__(256) gather_bench_kernel(const uint8_t* __restrict__ buf, uint64_t nrec,
                                                           uint32_t iters, uint32_t seed, uint32_t* sink) {
    uint32_t x = (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u ^ seed;
    uint32_t acc = 0;
    for (uint32_t it = 0; it < iters; it += 8) {
        uint32_t w[8][RB / 4 > 16 ? 16 : RB / 4];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            x ^= x << 13;
            x ^= x >> 17;
            x ^= x << 5;
            const uint64_t r = ((uint64_t)x * nrec) >> 32;
            ldg_record<RB>(buf + r * RB, w[u]);
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) acc ^= w[u][0] ^ w[u][RB / 4 - 1];
    }
    if (acc == 0x9E3779B9u) sink[0] = acc;
}

// ------------------------------------------------------------------------- launchers
cudaError_t launch_track(const TrackArgs& a, const TrackMode& m, int nfibres, bool half, int num_sms,
                         cudaStream_t st) {
    switch (nfibres * 2 + (half ? 1 : 0)) {
        case 2: return launch_track_f<1, false>(a, m, num_sms, st);
        case 3: return launch_track_f<1, true>(a, m, num_sms, st);
        case 4: return launch_track_f<2, false>(a, m, num_sms, st);
        case 5: return launch_track_f<2, true>(a, m, num_sms, st);
        case 6: return launch_track_f<3, false>(a, m, num_sms, st);
        case 7: return launch_track_f<3, true>(a, m, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

RecLayout rec_layout(int nx, int ny, int nz, uint32_t b, bool margin) {
    RecLayout L;
    const uint32_t e = 1u << b;
    L.b = b;
    L.nbx = ((uint32_t)nx + e - 1u) >> b;
    L.nby = ((uint32_t)ny + e - 1u) >> b;
    L.nbz = ((uint32_t)nz + e - 1u) >> b;
    if (PT_REC_MARGIN && margin && b) {  // one brick of sentinels on every side
        L.nbx += 2u;
        L.nby += 2u;
        L.nbz += 2u;
        L.off = e;
    }
    return L;
}

cudaError_t launch_repack(const void* dyads, const void* f, const uint8_t* mask, uint8_t* rec,
                          int nx, int ny, int nz, const RecLayout& L, int S, int F, bool half, int rec_bytes,
                          unsigned long long* bad, unsigned long long* maxabs, cudaStream_t st) {
    const int64_t V = (int64_t)nx * ny * nz;
    const int64_t total = V * (int64_t)S;
    // bricked layouts: the padding of ragged edge bricks (and the margin bricks) holds
    // sentinel records (all-ones words: f0 = NaN pattern = outside the mask)
    if (L.b) {
        const cudaError_t e = cudaMemsetAsync(rec, 0xFF, (size_t)L.nvox() * (size_t)S * (size_t)rec_bytes, st);
        if (e != cudaSuccess) return e;
    }
    int64_t blocks = (total + 255) / 256;
    if (blocks > 148 * 64) blocks = 148 * 64;
    if (blocks < 1) blocks = 1;
    if (half)
        repack_kernel<true><<<(unsigned)blocks, 256, 0, st>>>(dyads, f, mask, rec, nx, ny, V, L, S, F, rec_bytes, bad, maxabs);
    else
        repack_kernel<false><<<(unsigned)blocks, 256, 0, st>>>(dyads, f, mask, rec, nx, ny, V, L, S, F, rec_bytes, bad, maxabs);
    return cudaGetLastError();
}

cudaError_t launch_map_sum(const uint32_t* map, int64_t V, unsigned long long* out, cudaStream_t st) {
    int64_t blocks = (V + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    map_sum_kernel<<<(unsigned)blocks, 256, 0, st>>>(map, V, out);
    return cudaGetLastError();
}

cudaError_t launch_map_unpermute(const uint32_t* scratch, uint32_t mask, bool rv_keys, int nx, int ny,
                                 const RecLayout& L, uint32_t* map, int64_t V, bool accumulate, cudaStream_t st) {
    if (V <= 0) return cudaSuccess;
    const int64_t blocks = (V + 255) / 256 < 4096 ? (V + 255) / 256 : 4096;
    map_unpermute_kernel<<<(unsigned)blocks, 256, 0, st>>>(scratch, mask, rv_keys, (uint32_t)nx, (uint32_t)ny, L, map,
                                                            V, accumulate);
    return cudaGetLastError();
}

int gather_bench_blocks_per_sm(int rec_bytes) {
    int per_sm = 0;
    switch (rec_bytes) {
        case 8: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<8>, 256, 0); break;
        case 16: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<16>, 256, 0); break;
        case 32: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<32>, 256, 0); break;
        case 64: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_bench_kernel<64>, 256, 0); break;
        default: break;
    }
    return per_sm;
}

cudaError_t launch_gather_bench(const uint8_t* buf, uint64_t nrec, int rec_bytes, uint32_t iters,
                                int blocks, uint32_t seed, uint32_t* sink, cudaStream_t st) {
    switch (rec_bytes) {
        case 8: gather_bench_kernel<8><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        case 16: gather_bench_kernel<16><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        case 32: gather_bench_kernel<32><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        case 64: gather_bench_kernel<64><<<blocks, 256, 0, st>>>(buf, nrec, iters, seed, sink); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

}  // namespace pt
