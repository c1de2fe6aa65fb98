// Shared device/host helpers of the CUDA path (never shared with oracle/).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace ipt {

// ------------------------------------------------------------------------------------
// Strength-reduced division by an invariant divisor (§4.4, :745-749: "computing
// a fixed-point reciprocal, and then converting integer division into a multiplication
// by the reciprocal followed by a shift [10]").  Granlund-Montgomery round-up variant for
// 32-bit unsigned dividends, exact for every x < 2^32 and 1 <= d < 2^32:
//   l = ceil(log2 d), mul = floor(2^32 (2^l - d) / d) + 1, s1 = min(l, 1), s2 = max(l-1, 0)
//   t = umulhi(mul, x),  q = (t + ((x - t) >> s1)) >> s2.
// ------------------------------------------------------------------------------------
struct FastDiv {
    uint32_t d, mul, s1, s2;
};

inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f;
    f.d = d;
    uint32_t l = 0;
    while (l < 32 && (uint64_t(1) << l) < d) ++l;
    uint64_t m = ((uint64_t(1) << 32) * ((uint64_t(1) << l) - d)) / d + 1;
    f.mul = static_cast<uint32_t>(m);
    f.s1 = l < 1 ? l : 1;
    f.s2 = l > 1 ? l - 1 : 0;
    return f;
}

__host__ __device__ __forceinline__ uint32_t fdiv(uint32_t x, const FastDiv &f) {
#ifdef __CUDA_ARCH__
    uint32_t t = __umulhi(f.mul, x);
#else
    uint32_t t = static_cast<uint32_t>((static_cast<uint64_t>(f.mul) * x) >> 32);
#endif
    return (t + ((x - t) >> f.s1)) >> f.s2;
}

__host__ __device__ __forceinline__ uint32_t fmod_(uint32_t x, const FastDiv &f) {
    return x - fdiv(x, f) * f.d;
}

// (x * y) mod d for x, y < d.  `wide` selects 64-bit arithmetic when d >= 2^16 (then
// x*y may not fit 32 bits); the narrow path is two IMADs and a strength-reduced mod.
__device__ __forceinline__ uint32_t mulmod(uint32_t x, uint32_t y, const FastDiv &f, bool wide) {
    if (!wide) return fmod_(x * y, f);
    return static_cast<uint32_t>((static_cast<uint64_t>(x) * y) % f.d);
}

// Opaque element words.
template <int EB> struct Word;
template <> struct Word<1> { using T = uint8_t; };
template <> struct Word<2> { using T = uint16_t; };
template <> struct Word<4> { using T = uint32_t; };
template <> struct Word<8> { using T = unsigned long long; };
template <> struct Word<16> { using T = uint4; };

// Streaming global accesses: data are touched once per pass, keep them out of L1.
__device__ __forceinline__ uint4 ldg16(const void *p) {
    uint4 v;
    asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ void stg16(void *p, const uint4 &v) {
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}

template <class T> __device__ __forceinline__ T ldg(const T *p) { return *p; }

// Cluster-wide barrier with release/acquire semantics (all threads of every CTA of the
// cluster must call it).  Orders every CTA's prior global reads before any CTA's
// subsequent global writes: the in-place hazard barrier of the column-tile kernels.
__device__ __forceinline__ void cluster_barrier() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
    asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
}

}  // namespace ipt
