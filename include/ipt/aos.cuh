// include/ipt/aos.cuh -- warp-cooperative Array-of-Structures loads and stores
// (§6.2, :1071-1105).  Header-only CUDA C++ for sm_100a.
//
// A warp whose 32 lanes each want one S-word struct from 32 consecutive structs reads the
// 32*S-word chunk with S fully coalesced 128-byte loads -- lane l's register k then holds
// chunk word k*32 + l -- and transposes the S x 32 register array in place so that lane
// l's register k holds word l*S + k, i.e. its own struct.  That register transposition
// is R2C(S, 32) (reading C16: rows = registers, columns = lanes, :1073), done with the
// paper's decomposition restricted to SIMD primitives:
//   * row permutation q / q^{-1} of the registers: static renaming (§6.2.3, :1083);
//   * column rotations p_j, r_j (lane-dependent amounts): branch-free barrel rotations,
//     ceil(log2 S) select steps (§6.2.2, :1081);
//   * row shuffle d'_i: one __shfl_sync per register (§6.2.1, :1075);
//   * S is a template constant, so c, a, b, the inverses and every per-register index are
//     compile-time (§6.2.4, :1085).
// The store is the inverse, C2R(S, 32), followed by S coalesced 128-byte stores.
//
//   warp_load_aos<S>(chunk, r):  all 32 lanes, chunk = first word of 32 consecutive
//                                structs (same pointer in every lane, 4-byte aligned);
//                                afterwards r[k] = chunk[lane*S + k].
//   warp_store_aos<S>(chunk, r): inverse: chunk[lane*S + k] = r[k].
//   warp_gather_aos<S>(base, idx, r) / warp_scatter_aos<S>(base, idx, r): random access,
//                                lane l's struct base[idx_l*S .. idx_l*S + S) (below).
//   coalesced_ptr<T>: Fig. 10 interface (:1089-1097): `T v = *cp;` / `*cp = v;`.  Uses the
//                     cooperative path when the whole warp is converged and the lanes'
//                     pointers are unit-stride (p_lane == p_0 + lane); otherwise a plain
//                     per-lane access.  sizeof(T) must be a multiple of 4, at most 128.
#pragma once

#include <cstdint>
#include <cstring>

namespace ipt {
namespace aos_detail {

constexpr int gcd_c(int x, int y) { return y == 0 ? x : gcd_c(y, x % y); }
// x^{-1} mod y for coprime x, y; 0 when y == 1 (reading C4).
constexpr int mmi_c(int x, int y) {
    if (y == 1) return 0;
    for (int k = 1; k < y; ++k)
        if ((x * k) % y == 1) return k;
    return 0;
}
constexpr int ilog2_ceil(int v) { return v <= 1 ? 0 : 1 + ilog2_ceil((v + 1) / 2); }
constexpr int log2_exact(int v) { return v <= 1 ? 0 : 1 + log2_exact(v / 2); }

// The S x 32 register array: M = S rows (registers), N = 32 columns (lanes).
template <int S>
struct Geo {
    static constexpr int M = S, N = 32;
    static constexpr int c = gcd_c(S, 32);  // a power of two dividing 32
    static constexpr int a = S / c, b = 32 / c;
    static constexpr int lb = log2_exact(b), lc = log2_exact(c);
    static constexpr int ainv = mmi_c(a % b, b);  // a^{-1} mod b
    static constexpr int binv = mmi_c(b % a, a);  // b^{-1} mod a
    static constexpr int steps = ilog2_ceil(S);
    // Eq. 33: q(i) = (i N - floor(i / a)) mod M
    static constexpr int q(int i) { return ((i * N - i / a) % M + M) % M; }
    // Eq. 34: q^{-1}(i) = (floor((c-1+i)/c) b^{-1}) mod a + (((c-1) i) mod c) a
    static constexpr int qinv(int i) { return (((c - 1 + i) / c) * binv) % a + (((c - 1) * i) % c) * a; }
};

// out[i] = r[(i + d) mod S] for a compile-time d, selected by `on` (one barrel stage).
template <int S, int D>
__device__ __forceinline__ void rotate_stage(uint32_t (&r)[S], bool on) {
    uint32_t t[S];
#pragma unroll
    for (int i = 0; i < S; ++i) t[i] = on ? r[(i + D) % S] : r[i];
#pragma unroll
    for (int i = 0; i < S; ++i) r[i] = t[i];
}

template <int S, int K>
__device__ __forceinline__ void barrel(uint32_t (&r)[S], int g) {
    if constexpr (K < Geo<S>::steps) {
        rotate_stage<S, (1 << K) % S>(r, (g >> K) & 1);
        barrel<S, K + 1>(r, g);
    }
}

// Gather rotation of one lane's registers: out[i] = r[(i + g) mod S], 0 <= g < S, as a
// branch-free barrel rotator (§6.2.2): ceil(log2 S) stages of S selects.
template <int S>
__device__ __forceinline__ void rotate(uint32_t (&r)[S], int g) {
    barrel<S, 0>(r, g);
}

// Static row permutation (§6.2.3): out[i] = r[f(i)] with f known at compile time.
template <int S, bool INV>
__device__ __forceinline__ void permute_rows(uint32_t (&r)[S]) {
    uint32_t t[S];
#pragma unroll
    for (int i = 0; i < S; ++i) t[i] = r[INV ? Geo<S>::qinv(i) : Geo<S>::q(i)];
#pragma unroll
    for (int i = 0; i < S; ++i) r[i] = t[i];
}

__device__ __forceinline__ int lane_id() {
    int l;
    asm("mov.u32 %0, %%laneid;" : "=r"(l));
    return l;
}

}  // namespace aos_detail

// In-register R2C(S, 32) (§4.3 gather forms, Eqs. 34, 35, 24, 36 with M = S,
// N = 32): lane j's register i receives word j*S + i of the chunk whose word i*32 + j it
// held.
template <int S>
__device__ __forceinline__ void r2c_registers(uint32_t (&r)[S]) {
    using G = aos_detail::Geo<S>;
    const int j = aos_detail::lane_id();
    // 1. gather q^{-1} (Eq. 34): static renaming.
    aos_detail::permute_rows<S, true>(r);
    // 2. gather p^{-1}_j(i) = (i - j) mod S (Eq. 35): lane-dependent rotation.
    aos_detail::rotate<S>(r, (S - j % S) % S);
    // 3. row gather d'_i(j) = ((i + floor(j/b)) mod S + j S) mod 32 (Eq. 24): shuffles.
#pragma unroll
    for (int i = 0; i < S; ++i) {
        int t = i + (j >> G::lb);
        t = t >= S ? t - S : t;
        const int src = (t + j * S) & 31;
        r[i] = __shfl_sync(0xffffffffu, r[i], src);
    }
    // 4. [c > 1] gather r^{-1}_j(i) = (i - floor(j/b)) mod S (Eq. 36).
    if (G::c > 1) aos_detail::rotate<S>(r, (S - (j >> G::lb) % S) % S);
}

// In-register C2R(S, 32) (§4.2 gather forms, Eqs. 23, 31, 32, 33): the inverse.
template <int S>
__device__ __forceinline__ void c2r_registers(uint32_t (&r)[S]) {
    using G = aos_detail::Geo<S>;
    const int j = aos_detail::lane_id();
    // 1. [c > 1] gather r_j(i) = (i + floor(j/b)) mod S (Eq. 23).
    if (G::c > 1) aos_detail::rotate<S>(r, (j >> G::lb) % S);
    // 2. row gather d'^{-1}_i(j) (Eq. 31, closed form of DESIGN.md §2):
    //    q = (j - i) mod 32, l = q mod c, h = (a^{-1} floor(q/c) + [i + l >= S]) mod b.
#pragma unroll
    for (int i = 0; i < S; ++i) {
        const int q = (j - i) & 31;
        const int l = q & (G::c - 1);
        int h = (G::ainv * (q >> G::lc)) & (G::b - 1);
        if (i + l >= S) h = (h + 1) & (G::b - 1);
        r[i] = __shfl_sync(0xffffffffu, r[i], l * G::b + h);
    }
    // 3. gather p_j(i) = (i + j) mod S (Eq. 32).
    aos_detail::rotate<S>(r, j % S);
    // 4. gather q (Eq. 33): static renaming.
    aos_detail::permute_rows<S, false>(r);
}

template <int S>
__device__ __forceinline__ void warp_load_aos(const uint32_t *chunk, uint32_t (&r)[S]) {
    const int j = aos_detail::lane_id();
#pragma unroll
    for (int k = 0; k < S; ++k) r[k] = chunk[k * 32 + j];  // S coalesced 128-byte loads
    r2c_registers<S>(r);
}

template <int S>
__device__ __forceinline__ void warp_store_aos(uint32_t *chunk, uint32_t (&r)[S]) {
    const int j = aos_detail::lane_id();
    c2r_registers<S>(r);
#pragma unroll
    for (int k = 0; k < S; ++k) chunk[k * 32 + j] = r[k];  // S coalesced 128-byte stores
}

// Random-access AoS gather / scatter (SURVEY §8 row f1; PAPER.md :1087, :1099, Fig. 9):
// lane l wants struct idx_l (any index, repeats allowed for the gather) of an S-word AoS
// array.  The 32 structs are treated as one virtual contiguous 32*S-word chunk: virtual
// word v = k*32 + l is word (v mod S) of lane (v / S)'s struct, whose index the warp
// exchanges with one __shfl_sync per register ("shuffle indices across lanes"); register k
// of lane l loads it, so each load instruction fetches whole structs cooperatively (32/S
// structs, their words contiguous) instead of one word of 32 scattered structs.  The
// register array is then exactly the unit-stride chunk of warp_load_aos, and R2C(S, 32)
// hands lane l its struct.  The scatter is the inverse (C2R(S, 32), then the cooperative
// stores); with repeated indices the stored value is that of one of the lanes.
//   warp_gather_aos<S>(base, idx, r):  r[k] = base[idx * S + k]   (all 32 lanes)
//   warp_scatter_aos<S>(base, idx, r): base[idx * S + k] = r[k]
template <int S>
__device__ __forceinline__ void warp_gather_aos(const uint32_t *base, uint32_t idx, uint32_t (&r)[S]) {
    const int j = aos_detail::lane_id();
#pragma unroll
    for (int k = 0; k < S; ++k) {
        const int v = k * 32 + j;  // virtual word: word v % S of the struct of lane v / S
        const uint32_t owner_idx = __shfl_sync(0xffffffffu, idx, v / S);
        r[k] = base[static_cast<uint64_t>(owner_idx) * S + (v % S)];
    }
    r2c_registers<S>(r);
}

template <int S>
__device__ __forceinline__ void warp_scatter_aos(uint32_t *base, uint32_t idx, uint32_t (&r)[S]) {
    const int j = aos_detail::lane_id();
    c2r_registers<S>(r);
#pragma unroll
    for (int k = 0; k < S; ++k) {
        const int v = k * 32 + j;
        const uint32_t owner_idx = __shfl_sync(0xffffffffu, idx, v / S);
        base[static_cast<uint64_t>(owner_idx) * S + (v % S)] = r[k];
    }
}

// Fig. 10: `coalesced_ptr<T> c_ptr(ptr); T v = *c_ptr; *c_ptr = v;`
template <class T>
struct coalesced_ptr {
    static_assert(sizeof(T) % 4 == 0 && sizeof(T) <= 128, "coalesced_ptr: sizeof(T) must be 4k <= 128");
    static constexpr int S = static_cast<int>(sizeof(T) / 4);
    T *p;

    __device__ explicit coalesced_ptr(T *ptr) : p(ptr) {}

    // Warp-uniform: every lane active and p_lane == p_0 + lane, p_0 4-byte aligned.  Structs
    // of at most 16 bytes take the per-lane path: B200's coalescer already merges a warp's
    // <= 512 contiguous bytes, and the round-1 Fig. 8 measurement (profiles/r01_aos_config4)
    // shows the transposition only pays from 20-byte structs on.
    __device__ __forceinline__ bool cooperative() const {
        if constexpr (S <= 4) return false;
        if (__activemask() != 0xffffffffu) return false;
        const unsigned long long u = reinterpret_cast<unsigned long long>(p);
        const unsigned long long u0 = __shfl_sync(0xffffffffu, u, 0);
        const int j = aos_detail::lane_id();
        return __all_sync(0xffffffffu, u == u0 + static_cast<unsigned long long>(j) * sizeof(T) && (u0 & 3) == 0);
    }
    __device__ __forceinline__ T load() const {
        if (cooperative()) {
            uint32_t r[S];
            warp_load_aos<S>(reinterpret_cast<const uint32_t *>(p - aos_detail::lane_id()), r);
            T v;
            memcpy(&v, r, sizeof(T));
            return v;
        }
        return *p;
    }
    __device__ __forceinline__ void store(const T &v) {
        if (cooperative()) {
            uint32_t r[S];
            memcpy(r, &v, sizeof(T));
            warp_store_aos<S>(reinterpret_cast<uint32_t *>(p - aos_detail::lane_id()), r);
            return;
        }
        *p = v;
    }
    __device__ __forceinline__ operator T() const { return load(); }
    __device__ __forceinline__ coalesced_ptr &operator=(const T &v) {
        store(v);
        return *this;
    }
    __device__ __forceinline__ coalesced_ptr &operator*() { return *this; }
};

}  // namespace ipt
