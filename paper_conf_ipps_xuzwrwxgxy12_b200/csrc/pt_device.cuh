// pt_device.cuh -- device-side building blocks of the tracking kernels (sm_100a).
//
// Every floating-point operation of the stepping arithmetic is written with __fmul_rn /
// __fadd_rn / __fsub_rn (one IEEE binary32 operation, round-to-nearest-even, never
// contracted into an FMA) and the library is additionally compiled with -fmad=false, so
// the results are bit-identical to any correctly rounded binary32 evaluation of the same
// expression order (R15 in DESIGN.md).  Citations: P:Lnnn = PAPER.md line.
#pragma once
#include <cstdint>
#include <cuda_fp16.h>

namespace pt {

constexpr uint32_t kFull = 0xFFFFFFFFu;

// ---------------------------------------------------------------------------- RNG (R16)
// Philox4x32-10 (Salmon et al., SC'11): counter-based, so a particle's draws depend only
// on (rng_seed, pid, stream, block) and never on scheduling.  Counter = {block, pid_lo,
// pid_hi, stream}.  Stream 0 (1 = the reverse half of a bidirectional streamline, R22):
// words 0..2 of block b give the sample indices of steps 3b, 3b+1, 3b+2; word 3 of block 0
// gives the first step's sign.  Stream 2 + half, block n: interpolation draws of step n
// (R23) and the first-fibre draw (word 3 of block 0, R24).  Replaces the combined
// Tausworthe generator of P:L153 (the frozen contract: DESIGN.md R16).
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        if (r) {
            k0 += 0x9E3779B9u;
            k1 += 0xBB67AE85u;
        }
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
    }
    return c;
}

// sample index s = floor(w * S / 2^32) (integer only; R16)
__device__ __forceinline__ uint32_t sample_of(uint32_t w, uint32_t S) { return __umulhi(w, S); }

// ---------------------------------------------------------------------------- records
// One record per (voxel, sample): the F fibres' unit vector and fraction (the sample
// volumes of P:L125 / Fig. 1, repacked).  fp32: {x,y,z,f} x F (16 B per fibre,
// padded to 16/32/64 B); fp16: {x,y,z,f} halves x F (8 B per fibre, padded to 8/16/32 B).
// A voxel outside the mask carries the sentinel f0 = all-ones (a NaN that validated
// input never contains) in every sample: the gather that fetches the next step's record
// is also the mask test of the candidate voxel (R11).
template <int F, bool HALF>
struct Rec {
    static constexpr int kRaw = HALF ? 8 * F : 16 * F;
    static constexpr int kBytes = kRaw <= 8 ? 8 : kRaw <= 16 ? 16 : kRaw <= 32 ? 32 : 64;
    static constexpr int kWords = kBytes / 4;
    uint32_t w[kWords];

    __device__ __forceinline__ bool outside() const {
        return HALF ? ((w[1] >> 16) == 0xFFFFu) : (w[3] == 0xFFFFFFFFu);
    }
    // exchange fibre js (< F) with fibre 0 (straight-line selects, no local memory)
    __device__ __forceinline__ void swap_to_front(int js) {
        constexpr int WF = HALF ? 2 : 4;  // words per fibre
#pragma unroll
        for (int j = 1; j < F; ++j) {
            const bool p = js == j;
#pragma unroll
            for (int k = 0; k < WF; ++k) {
                const uint32_t a = w[k], b = w[WF * j + k];
                w[k] = p ? b : a;
                w[WF * j + k] = p ? a : b;
            }
        }
    }
    __device__ __forceinline__ void fibre(int j, float& x, float& y, float& z, float& f) const {
        if (HALF) {
            const uint32_t a = w[2 * j], b = w[2 * j + 1];
            x = __half2float(__ushort_as_half((unsigned short)(a & 0xFFFFu)));
            y = __half2float(__ushort_as_half((unsigned short)(a >> 16)));
            z = __half2float(__ushort_as_half((unsigned short)(b & 0xFFFFu)));
            f = __half2float(__ushort_as_half((unsigned short)(b >> 16)));
        } else {
            x = __uint_as_float(w[4 * j + 0]);
            y = __uint_as_float(w[4 * j + 1]);
            z = __uint_as_float(w[4 * j + 2]);
            f = __uint_as_float(w[4 * j + 3]);
        }
    }
};

// ---------------------------------------------------------------------------- direction
// Direction of the last step, d = sign * (a record's unit vector).  fp32 records: three
// floats.  fp16 records: d is a sign-flipped binary16 vector, kept packed (xy = x | y << 16,
// z in the low half of zw) and never decoded for the dot products of the fibre choice:
// they run as mixed-precision FMAs (FHFMA: f32 = f16 * f16 + f32).  The product of two
// binary16 values is exact in binary32 (22 significand bits, exponents within range), so
// fma(a, b, c) = round(a*b + c) is bit-identical to the contract's round(round(a*b) + c)
// (R15); the first product is added to -0, which returns it unchanged, signed zero included.
__device__ __forceinline__ float hfma_lo(uint32_t a, uint32_t b, float c) {
    float d;
    asm("{.reg .f16 ha, hb;\n\tmov.b32 {ha, _}, %1;\n\tmov.b32 {hb, _}, %2;\n\tfma.rn.f32.f16 %0, ha, hb, %3;\n\t}"
        : "=f"(d) : "r"(a), "r"(b), "f"(c));
    return d;
}
__device__ __forceinline__ float hfma_hi(uint32_t a, uint32_t b, float c) {
    float d;
    asm("{.reg .f16 ha, hb;\n\tmov.b32 {_, ha}, %1;\n\tmov.b32 {_, hb}, %2;\n\tfma.rn.f32.f16 %0, ha, hb, %3;\n\t}"
        : "=f"(d) : "r"(a), "r"(b), "f"(c));
    return d;
}
// ((vx * dx + vy * dy) + vz * dz) of a packed fp16 vector (w_xy, w_z) and a packed direction
__device__ __forceinline__ float hdot(uint32_t wxy, uint32_t wz, uint32_t dxy, uint32_t dz) {
    return hfma_lo(wz, dz, hfma_hi(wxy, dxy, hfma_lo(wxy, dxy, -0.f)));
}
__device__ __forceinline__ float half_lo(uint32_t w) { return __half2float(__ushort_as_half((unsigned short)(w & 0xFFFFu))); }
__device__ __forceinline__ float half_hi(uint32_t w) { return __half2float(__ushort_as_half((unsigned short)(w >> 16))); }

// Random gather of one record through the read-only (texture/L1) path: one LDG of 8, 16
// or 32 bytes (two 32-B LDGs for a 64-B record).
template <int BYTES>
__device__ __forceinline__ void ldg_record(const void* p, uint32_t* w);

template <>
__device__ __forceinline__ void ldg_record<8>(const void* p, uint32_t* w) {
    asm("ld.global.nc.v2.b32 {%0,%1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "l"(p));
}
template <>
__device__ __forceinline__ void ldg_record<16>(const void* p, uint32_t* w) {
    asm("ld.global.nc.v4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3])
                 : "l"(p));
}
template <>
__device__ __forceinline__ void ldg_record<32>(const void* p, uint32_t* w) {
    asm("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]),
                   "=r"(w[6]), "=r"(w[7])
                 : "l"(p));
}
template <>
__device__ __forceinline__ void ldg_record<64>(const void* p, uint32_t* w) {
    ldg_record<32>(p, w);
    ldg_record<32>(static_cast<const char*>(p) + 32, w + 8);
}

// Predicated variants for straight-line step code: the load / reduction is issued only by
// lanes with p != 0; the destination registers of the other lanes keep their values.
template <int BYTES>
__device__ __forceinline__ void ldg_record_if(bool p, const void* ptr, uint32_t* w);

template <>
__device__ __forceinline__ void ldg_record_if<8>(bool p, const void* ptr, uint32_t* w) {
    asm("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %3, 0;\n\t@q ld.global.nc" ".v2.b32 {%0,%1}, [%2];\n\t}"
        : "+r"(w[0]), "+r"(w[1])
        : "l"(ptr), "r"((int)p));
}
template <>
__device__ __forceinline__ void ldg_record_if<16>(bool p, const void* ptr, uint32_t* w) {
    asm("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %5, 0;\n\t@q ld.global.nc" ".v4.b32 {%0,%1,%2,%3}, [%4];\n\t}"
        : "+r"(w[0]), "+r"(w[1]), "+r"(w[2]), "+r"(w[3])
        : "l"(ptr), "r"((int)p));
}
template <>
__device__ __forceinline__ void ldg_record_if<32>(bool p, const void* ptr, uint32_t* w) {
    asm("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %9, 0;\n\t@q ld.global.nc" ".v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n\t}"
        : "+r"(w[0]), "+r"(w[1]), "+r"(w[2]), "+r"(w[3]), "+r"(w[4]), "+r"(w[5]), "+r"(w[6]), "+r"(w[7])
        : "l"(ptr), "r"((int)p));
}
template <>
__device__ __forceinline__ void ldg_record_if<64>(bool p, const void* ptr, uint32_t* w) {
    ldg_record_if<32>(p, ptr, w);
    ldg_record_if<32>(p, static_cast<const char*>(ptr) + 32, w + 8);
}

#ifndef PT_RED_EVICT_LAST
#define PT_RED_EVICT_LAST 0  // experiment: map REDs with an L2 evict_last cache policy
#endif
__device__ __forceinline__ void red_add_if(bool p, uint32_t* addr, uint32_t v) {
#if PT_RED_EVICT_LAST
    asm volatile("{\n\t.reg .pred q;\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
                 "setp.ne.b32 q, %2, 0;\n\t@q red.global.add.L2::cache_hint.u32 [%0], %1, pol;\n\t}"
                 :: "l"(addr), "r"(v), "r"((int)p) : "memory");
#else
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q red.global.add.u32 [%0], %1;\n\t}"
                 :: "l"(addr), "r"(v), "r"((int)p) : "memory");
#endif
}

// ---------------------------------------------------------------------------- lookup (R10)
// Centred coordinates q = x - c, c = floor(N/2); index = c + trunc(q) - signbit(q):
// voxel i covers [i-c, i-c+1) for i >= c and (i-c, i-c+1] for i < c.
__device__ __forceinline__ int axis_index(float q, int c) {
    return c + __float2int_rz(q) - (int)(__float_as_uint(q) >> 31);
}

// ---------------------------------------------------------------------------- record layout
// Position of voxel (ix, iy, iz) in the record volume.  Bricked layout: the volume is cut
// into bricks of 2^b x 2^b x 2^b voxels (bricks raster-ordered, nbx x nby per z-slab of
// bricks; voxels raster-ordered inside a brick), so the records of a 3-D neighbourhood --
// everything a tract touches over a few steps -- sit in a few contiguous MB instead of
// being strided by whole planes (fewer DRAM pages and TLB entries per neighbourhood).
// b = 0 is the plain raster layout (nbx = nx, nby = ny).  Layout only: which record a
// step reads is unchanged, so results are unaffected.
__device__ __forceinline__ uint32_t rec_vox(int ix, int iy, int iz, uint32_t b, uint32_t nbx, uint32_t nby,
                                            uint32_t off = 0u) {
    const uint32_t m = (1u << b) - 1u;
    const uint32_t x = (uint32_t)ix + off, y = (uint32_t)iy + off, z = (uint32_t)iz + off;
    const uint32_t br = ((z >> b) * nby + (y >> b)) * nbx + (x >> b);
    return (br << (3u * b)) | ((z & m) << (2u * b)) | ((y & m) << b) | (x & m);
}
// Index of record (voxel rv of the record order, sample s): voxel-major, a voxel's S samples
// contiguous (a sample-major order inside each brick, which puts a voxel's samples on
// different L2 slices, measured 3.7-6 % slower: DESIGN §11).
__host__ __device__ __forceinline__ uint64_t rec_slot(uint32_t rv, uint32_t s, uint32_t S, uint32_t b) {
    (void)b;
    return (uint64_t)rv * S + s;
}
// the same from a raster voxel index (variant / ablation kernels, repack)
__device__ __forceinline__ uint32_t rec_vox_raster(uint32_t v, uint32_t nx, uint32_t ny, uint32_t b, uint32_t nbx,
                                                   uint32_t nby, uint32_t off = 0u) {
    if (b == 0u) return v;
    const uint32_t z = v / (nx * ny), r = v - z * (nx * ny), y = r / nx, x = r - y * nx;
    return rec_vox((int)x, (int)y, (int)z, b, nbx, nby, off);
}

}  // namespace pt
