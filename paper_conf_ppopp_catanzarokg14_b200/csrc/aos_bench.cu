// Consumer kernels of the warp-cooperative AoS helpers (include/ipt/aos.cuh; SURVEY §8
// row a6, BASELINE config 4; §6.2 Figs. 8-10).  Exported through
// include/ipt_debug.h for the parity tests and the config-4 benchmark:
//   * copy  (dst[k] = src[k]) and store-only (dst[k] = f(k)) over `count` structs of S words;
//   * variants (the three lines of Fig. 8): DIRECT -- compiler-generated per-lane struct
//     access; VECTOR -- the widest native vector type that divides the struct; COALESCED --
//     coalesced_ptr<T> (in-register R2C/C2R);
//   * register dumps of warp_load_aos / warp_store_aos for the parity tests.
#include "ipt.h"
#include "ipt_debug.h"
#include "ipt/aos.cuh"
#include "plan.h"

namespace ipt {
namespace {

template <int S>
struct alignas(4) Words {
    uint32_t w[S];
};

// Store-only payload: word i of struct k is k * S + i (so dst ends up as 0, 1, 2, ...).
template <int S>
__device__ __forceinline__ Words<S> payload(int64_t k) {
    Words<S> v;
#pragma unroll
    for (int i = 0; i < S; ++i) v.w[i] = static_cast<uint32_t>(k * S + i);
    return v;
}

template <int S> struct VecOf { using V = uint32_t; };
template <int S> requires(S % 4 == 0) struct VecOf<S> { using V = uint4; };
template <int S> requires(S % 4 == 2) struct VecOf<S> { using V = uint2; };

template <int S>
__device__ __forceinline__ void vec_copy(const Words<S> *src, Words<S> *dst) {
    using V = typename VecOf<S>::V;
    constexpr int NV = static_cast<int>(sizeof(Words<S>) / sizeof(V));
    const V *s = reinterpret_cast<const V *>(src);
    V *d = reinterpret_cast<V *>(dst);
    V t[NV];
#pragma unroll
    for (int x = 0; x < NV; ++x) t[x] = s[x];
#pragma unroll
    for (int x = 0; x < NV; ++x) d[x] = t[x];
}
template <int S>
__device__ __forceinline__ void vec_store(Words<S> *dst, const Words<S> &v) {
    using V = typename VecOf<S>::V;
    constexpr int NV = static_cast<int>(sizeof(Words<S>) / sizeof(V));
    V *d = reinterpret_cast<V *>(dst);
    const V *s = reinterpret_cast<const V *>(&v);
#pragma unroll
    for (int x = 0; x < NV; ++x) d[x] = s[x];
}

// Grid-stride over whole warps of structs so that warps stay converged (the coalesced
// path needs all 32 lanes); the tail warp runs the fallback per-lane access.
template <int S, int VARIANT, bool COPY>
__global__ void __launch_bounds__(256) aos_kernel(const Words<S> *src, Words<S> *dst, int64_t count) {
    const int64_t nthreads = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t k = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k - (threadIdx.x & 31) < count;
         k += nthreads) {
        if (k >= count) continue;  // only in the tail warp
        if (VARIANT == IPT_AOS_DIRECT) {
            if (COPY) dst[k] = src[k];
            else dst[k] = payload<S>(k);
        } else if (VARIANT == IPT_AOS_VECTOR) {
            if (COPY) vec_copy<S>(src + k, dst + k);
            else vec_store<S>(dst + k, payload<S>(k));
        } else {
            coalesced_ptr<Words<S>> out(dst + k);
            if (COPY) {
                coalesced_ptr<Words<S>> in(const_cast<Words<S> *>(src + k));
                *out = static_cast<Words<S>>(*in);
            } else {
                *out = payload<S>(k);
            }
        }
    }
}

// Random access (Fig. 9): gather dst[k] = src[idx[k]] / scatter
// dst[idx[k]] = src[k].  DIRECT: per-lane struct access (compiler-generated); COALESCED:
// warp_gather_aos + warp_store_aos / warp_load_aos + warp_scatter_aos on whole warps, the
// tail warp per lane.  (VECTOR is treated as DIRECT with native vectors.)
template <int S, int VARIANT, bool GATHER>
__global__ void __launch_bounds__(256) aos_random_kernel(const Words<S> *src, const uint32_t *idx, Words<S> *dst,
                                                         int64_t count) {
    const int64_t nthreads = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t k = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k - (threadIdx.x & 31) < count;
         k += nthreads) {
        const int64_t k0 = k - (threadIdx.x & 31);
        if (VARIANT == IPT_AOS_COALESCED && k0 + 32 <= count) {  // whole warp: cooperative
            uint32_t r[S];
            const uint32_t j = idx[k];
            if (GATHER) {
                warp_gather_aos<S>(reinterpret_cast<const uint32_t *>(src), j, r);
                warp_store_aos<S>(reinterpret_cast<uint32_t *>(dst + k0), r);
            } else {
                warp_load_aos<S>(reinterpret_cast<const uint32_t *>(src + k0), r);
                warp_scatter_aos<S>(reinterpret_cast<uint32_t *>(dst), j, r);
            }
            continue;
        }
        if (k >= count) continue;
        const uint32_t j = idx[k];
        if (VARIANT == IPT_AOS_VECTOR) {
            if (GATHER) vec_copy<S>(src + j, dst + k);
            else vec_copy<S>(src + k, dst + j);
        } else {
            if (GATHER) dst[k] = src[j];
            else dst[j] = src[k];
        }
    }
}

template <int S>
cudaError_t run_random(const void *src, const uint32_t *idx, void *dst, int64_t count, int variant, bool gather,
                       cudaStream_t st);

// warp_load_aos dump: chunk c of 32 structs -> dump[c*32*S + lane*S + k] = r[k].
template <int S>
__global__ void warp_load_dump_kernel(const uint32_t *src, uint32_t *dump, int64_t nchunks) {
    const int64_t warp = (static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= nchunks) return;
    uint32_t r[S];
    warp_load_aos<S>(src + warp * 32 * S, r);
#pragma unroll
    for (int k = 0; k < S; ++k) dump[warp * 32 * S + lane * S + k] = r[k];
}

// warp_store_aos: lane l's registers are read per-lane from regs[c*32*S + l*S + k], then
// stored cooperatively into dst (must reproduce regs).
template <int S>
__global__ void warp_store_kernel(const uint32_t *regs, uint32_t *dst, int64_t nchunks) {
    const int64_t warp = (static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= nchunks) return;
    uint32_t r[S];
#pragma unroll
    for (int k = 0; k < S; ++k) r[k] = regs[warp * 32 * S + lane * S + k];
    warp_store_aos<S>(dst + warp * 32 * S, r);
}

int grid_for(int64_t count) {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t g = (count + 255) / 256;
    const int64_t cap = static_cast<int64_t>(sms) * 8;
    return static_cast<int>(g < cap ? (g < 1 ? 1 : g) : cap);
}

template <int S>
cudaError_t run_aos(const void *src, void *dst, int64_t count, int variant, bool copy, cudaStream_t st) {
    const auto *s = static_cast<const Words<S> *>(src);
    auto *d = static_cast<Words<S> *>(dst);
    const int grid = grid_for(count);
#define IPT_AOS_LAUNCH(V, C) aos_kernel<S, V, C><<<grid, 256, 0, st>>>(s, d, count)
    if (copy) {
        if (variant == IPT_AOS_DIRECT) IPT_AOS_LAUNCH(IPT_AOS_DIRECT, true);
        else if (variant == IPT_AOS_VECTOR) IPT_AOS_LAUNCH(IPT_AOS_VECTOR, true);
        else IPT_AOS_LAUNCH(IPT_AOS_COALESCED, true);
    } else {
        if (variant == IPT_AOS_DIRECT) IPT_AOS_LAUNCH(IPT_AOS_DIRECT, false);
        else if (variant == IPT_AOS_VECTOR) IPT_AOS_LAUNCH(IPT_AOS_VECTOR, false);
        else IPT_AOS_LAUNCH(IPT_AOS_COALESCED, false);
    }
#undef IPT_AOS_LAUNCH
    return cudaGetLastError();
}

template <int S>
cudaError_t run_dump(const void *in, void *out, int64_t nchunks, bool load, cudaStream_t st) {
    const int64_t threads = nchunks * 32;
    const unsigned grid = static_cast<unsigned>((threads + 255) / 256);
    if (load)
        warp_load_dump_kernel<S><<<grid, 256, 0, st>>>(static_cast<const uint32_t *>(in), static_cast<uint32_t *>(out),
                                                      nchunks);
    else
        warp_store_kernel<S><<<grid, 256, 0, st>>>(static_cast<const uint32_t *>(in), static_cast<uint32_t *>(out),
                                                  nchunks);
    return cudaGetLastError();
}

int grid_for(int64_t count);

template <int S>
cudaError_t run_random(const void *src, const uint32_t *idx, void *dst, int64_t count, int variant, bool gather,
                       cudaStream_t st) {
    const auto *s = static_cast<const Words<S> *>(src);
    auto *d = static_cast<Words<S> *>(dst);
    const int grid = grid_for(count);
#define IPT_AOS_RLAUNCH(V, G) aos_random_kernel<S, V, G><<<grid, 256, 0, st>>>(s, idx, d, count)
    if (gather) {
        if (variant == IPT_AOS_DIRECT) IPT_AOS_RLAUNCH(IPT_AOS_DIRECT, true);
        else if (variant == IPT_AOS_VECTOR) IPT_AOS_RLAUNCH(IPT_AOS_VECTOR, true);
        else IPT_AOS_RLAUNCH(IPT_AOS_COALESCED, true);
    } else {
        if (variant == IPT_AOS_DIRECT) IPT_AOS_RLAUNCH(IPT_AOS_DIRECT, false);
        else if (variant == IPT_AOS_VECTOR) IPT_AOS_RLAUNCH(IPT_AOS_VECTOR, false);
        else IPT_AOS_RLAUNCH(IPT_AOS_COALESCED, false);
    }
#undef IPT_AOS_RLAUNCH
    return cudaGetLastError();
}

template <int... Ss>
struct Dispatch;
template <>
struct Dispatch<> {
    static cudaError_t aos(int, const void *, void *, int64_t, int, bool, cudaStream_t) { return cudaErrorInvalidValue; }
    static cudaError_t random(int, const void *, const uint32_t *, void *, int64_t, int, bool, cudaStream_t) {
        return cudaErrorInvalidValue;
    }
    static cudaError_t dump(int, const void *, void *, int64_t, bool, cudaStream_t) { return cudaErrorInvalidValue; }
};
template <int S0, int... Ss>
struct Dispatch<S0, Ss...> {
    static cudaError_t aos(int S, const void *a, void *b, int64_t n, int v, bool c, cudaStream_t st) {
        return S == S0 ? run_aos<S0>(a, b, n, v, c, st) : Dispatch<Ss...>::aos(S, a, b, n, v, c, st);
    }
    static cudaError_t random(int S, const void *a, const uint32_t *ix, void *b, int64_t n, int v, bool g,
                              cudaStream_t st) {
        return S == S0 ? run_random<S0>(a, ix, b, n, v, g, st) : Dispatch<Ss...>::random(S, a, ix, b, n, v, g, st);
    }
    static cudaError_t dump(int S, const void *a, void *b, int64_t n, bool l, cudaStream_t st) {
        return S == S0 ? run_dump<S0>(a, b, n, l, st) : Dispatch<Ss...>::dump(S, a, b, n, l, st);
    }
};
using AllS = Dispatch<1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11, 12, 13, 14, 15, 16, 17, 18, 19, 20, 21, 22, 23, 24, 25,
                      26, 27, 28, 29, 30, 31, 32>;

ipt_status_t to_status(cudaError_t e) {
    if (e == cudaSuccess) return IPT_OK;
    cudaGetLastError();
    return e == cudaErrorInvalidValue ? IPT_ERR_INVALID_ARGUMENT : IPT_ERR_CUDA;
}

}  // namespace
}  // namespace ipt

extern "C" {

ipt_status_t ipt_debug_aos_copy(const void *src, void *dst, int64_t count, int words, int variant, void *stream) {
    if (!src || !dst || count < 0 || words < 1 || words > 32 || variant < 0 || variant > 2)
        return IPT_ERR_INVALID_ARGUMENT;
    if (count == 0) return IPT_OK;
    return ipt::to_status(ipt::AllS::aos(words, src, dst, count, variant, true, static_cast<cudaStream_t>(stream)));
}

ipt_status_t ipt_debug_aos_fill(void *dst, int64_t count, int words, int variant, void *stream) {
    if (!dst || count < 0 || words < 1 || words > 32 || variant < 0 || variant > 2) return IPT_ERR_INVALID_ARGUMENT;
    if (count == 0) return IPT_OK;
    return ipt::to_status(ipt::AllS::aos(words, nullptr, dst, count, variant, false, static_cast<cudaStream_t>(stream)));
}

ipt_status_t ipt_debug_aos_gather(const void *src, const uint32_t *idx, void *dst, int64_t count, int words,
                                  int variant, void *stream) {
    if (!src || !idx || !dst || count < 0 || words < 1 || words > 32 || variant < 0 || variant > 2)
        return IPT_ERR_INVALID_ARGUMENT;
    if (count == 0) return IPT_OK;
    return ipt::to_status(
        ipt::AllS::random(words, src, idx, dst, count, variant, true, static_cast<cudaStream_t>(stream)));
}

ipt_status_t ipt_debug_aos_scatter(const void *src, const uint32_t *idx, void *dst, int64_t count, int words,
                                   int variant, void *stream) {
    if (!src || !idx || !dst || count < 0 || words < 1 || words > 32 || variant < 0 || variant > 2)
        return IPT_ERR_INVALID_ARGUMENT;
    if (count == 0) return IPT_OK;
    return ipt::to_status(
        ipt::AllS::random(words, src, idx, dst, count, variant, false, static_cast<cudaStream_t>(stream)));
}

ipt_status_t ipt_debug_warp_load_dump(const void *src, void *dump, int64_t nchunks, int words, void *stream) {
    if (!src || !dump || nchunks < 0 || words < 1 || words > 32) return IPT_ERR_INVALID_ARGUMENT;
    if (nchunks == 0) return IPT_OK;
    return ipt::to_status(ipt::AllS::dump(words, src, dump, nchunks, true, static_cast<cudaStream_t>(stream)));
}

ipt_status_t ipt_debug_warp_store(const void *regs, void *dst, int64_t nchunks, int words, void *stream) {
    if (!regs || !dst || nchunks < 0 || words < 1 || words > 32) return IPT_ERR_INVALID_ARGUMENT;
    if (nchunks == 0) return IPT_OK;
    return ipt::to_status(ipt::AllS::dump(words, regs, dst, nchunks, false, static_cast<cudaStream_t>(stream)));
}

}  // extern "C"
