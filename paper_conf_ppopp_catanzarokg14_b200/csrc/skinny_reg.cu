// Skinny long-row shuffle in registers (SURVEY §8 rows a5 + a6; §6.1-6.2).
//
// The row shuffle of the skinny engine (skinny.cu) permutes a row of N = count elements by
// d'^{-1}_i.  Grouping the row's positions by n (x = t n + r, 0 <= r < n), the closed form
// of skinny.cu gives
//     d'^{-1}_i(t n + r) = lb_r + (h_r + t) mod b,   (lb_r, h_r) = d'^{-1}_i(r) split as l b + h,
// because x -> x + n keeps l and adds 1 to h (mod b).  So 32 consecutive n-element
// "structs" t = 32 g .. 32 g + 31 map, field by field, onto n runs of 32 consecutive
// positions: exactly the paper's SIMD AoS transposition (§6.2), with struct size S = n:
//   R2C (dst[d'^{-1}(x)] = src[x]):  warp_load_aos<S> of the 32 S-word chunk (S coalesced
//        128-byte loads + in-register R2C(S, 32)), then register k of lane l is stored at
//        position lb_k + (h_k + 32 g + l) mod b -- one coalesced 128-byte store per k;
//   C2R (dst[x] = src[d'^{-1}(x)]):  the mirror image with warp_store_aos<S>.
// No shared-memory staging of the data at all; 4-byte elements, S = n in 2..32 compiled
// as separate kernels.  The partial group at the end of the row (and, with the folded
// rotation, a group that straddles a column-block boundary) is moved element by element.
#include "ipt/aos.cuh"
#include "plan.h"

namespace ipt {
namespace {

constexpr int kRegThreads = 256;

__device__ __forceinline__ int32_t loc_src(const SkinnyRowParams &P, int DIR, int32_t rho) {
    int32_t L;
    if (DIR == ROW_R2C) {
        if (P.i == P.n - 1) return P.n;
        L = P.i + 1 + rho;
    } else {
        L = P.i + rho;
    }
    return L >= P.n ? L - P.n : L;
}
__device__ __forceinline__ int32_t loc_dst(const SkinnyRowParams &P, int DIR, int32_t rho) {
    int32_t L;
    if (DIR == ROW_R2C) {
        L = P.i + rho;
    } else {
        if (P.i == 0) return P.n;
        L = P.i - 1 + rho;
    }
    return L >= P.n ? L - P.n : L;
}

// d'^{-1}_i(x) = l b + h with q = (x - i) mod N, l = q mod c,
// h = (a^{-1} floor(q / c) + [i + l >= n]) mod b (skinny.cu, DESIGN.md §"Skinny engine").
__device__ __forceinline__ int64_t dpinv_pos(const SkinnyRowParams &P, int64_t x) {
    int64_t q = x - P.i;
    if (q < 0) q += P.N;
    const int64_t l = q % P.c;
    int64_t h = (P.ainv * (q / P.c)) % P.b;
    if (P.i + l >= P.n) h = h + 1 == P.b ? 0 : h + 1;
    return l * P.b + h;
}

template <int S, int DIR, bool FOLD>
__device__ __forceinline__ void skinny_reg_row(const SkinnyRowParams &P) {
    // U chunks per warp and iteration: all their loads are issued before any transposition
    // (memory-level parallelism for small S), U * S <= 32 data registers.
    constexpr int U = S <= 4 ? 8 : S <= 8 ? 4 : S <= 16 ? 2 : 1;
    __shared__ int2 s_lbh[S];  // (lb_k, h_k): one 8-byte shared load per run position
    __shared__ uint32_t *s_src[32], *s_dst[32];
    const int lane = threadIdx.x & 31;
    if (threadIdx.x < S) {
        const int64_t p = dpinv_pos(P, threadIdx.x);
        s_lbh[threadIdx.x] = make_int2(static_cast<int32_t>(p - p % P.b), static_cast<int32_t>(p % P.b));
    }
    const int nblk = FOLD ? P.c : 1;
    if (threadIdx.x < nblk) {
        const int32_t ls = loc_src(P, DIR, threadIdx.x), ld = loc_dst(P, DIR, threadIdx.x);
        // batches: matrix blockIdx.y of the launch, its own tmp row
        char *const Am = P.A + static_cast<int64_t>(blockIdx.y) * P.mat_stride;
        char *const tmpm = P.tmp + static_cast<int64_t>(blockIdx.y) * P.tmp_stride;
        s_src[threadIdx.x] = reinterpret_cast<uint32_t *>(ls == P.n ? tmpm : Am + ls * P.N * 4);
        s_dst[threadIdx.x] = reinterpret_cast<uint32_t *>(ld == P.n ? tmpm : Am + ld * P.N * 4);
    }
    __syncthreads();
    auto blk = [&](int64_t x) -> int32_t {
        return FOLD ? static_cast<int32_t>(fdiv(static_cast<uint32_t>(x), P.fd_b)) : 0;
    };
    const int32_t b = P.b;
    // run k of this row: positions lb_k + (h_k + t) mod b (t < b: one conditional subtract)
    auto run_pos = [&](int k, int32_t t) -> int32_t {
        const int2 lbh = s_lbh[k];
        int32_t y = lbh.y + t;
        y -= y >= b ? b : 0;
        return lbh.x + y;
    };
    const int32_t structs = static_cast<int32_t>(P.N / S);  // whole n-element groups of the row
    const int32_t groups = structs / 32;                     // whole warps' worth
    const int32_t warp = static_cast<int32_t>((static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5);
    const int32_t nwarps = static_cast<int32_t>((static_cast<int64_t>(gridDim.x) * blockDim.x) >> 5);
    uint32_t *src0 = s_src[0], *dst0 = s_dst[0];
    for (int32_t g0 = warp * U; g0 < groups; g0 += nwarps * U) {
        uint32_t r[U][S];
        if (DIR == ROW_R2C) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int32_t g = g0 + u;
                if (g >= groups) break;
                const int64_t x0 = static_cast<int64_t>(g) * 32 * S;
                const int32_t bs = blk(x0);
                if (!FOLD || blk(x0 + 32 * S - 1) == bs) {
                    const uint32_t *chunk = (FOLD ? s_src[bs] : src0) + x0;
#pragma unroll
                    for (int k = 0; k < S; ++k) r[u][k] = chunk[k * 32 + lane];  // coalesced
                } else {  // chunk straddles a column block: the same coalesced layout, per-word bases
#pragma unroll
                    for (int k = 0; k < S; ++k) {
                        const int64_t x = x0 + k * 32 + lane;
                        r[u][k] = s_src[blk(x)][x];
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int32_t g = g0 + u;
                if (g >= groups) break;
                r2c_registers<S>(r[u]);  // lane l now holds struct t = 32 g + l
                const int32_t t = g * 32 + lane;
#pragma unroll
                for (int k = 0; k < S; ++k) {
                    const int32_t y = run_pos(k, t);
                    (FOLD ? s_dst[blk(s_lbh[k].x)] : dst0)[y] = r[u][k];
                }
            }
        } else {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int32_t g = g0 + u;
                if (g >= groups) break;
                const int32_t t = g * 32 + lane;
#pragma unroll
                for (int k = 0; k < S; ++k) r[u][k] = (FOLD ? s_src[blk(s_lbh[k].x)] : src0)[run_pos(k, t)];
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int32_t g = g0 + u;
                if (g >= groups) break;
                c2r_registers<S>(r[u]);  // lane l's register k -> chunk word k * 32 + l
                const int64_t x0 = static_cast<int64_t>(g) * 32 * S;
                const int32_t bd = blk(x0);
                if (!FOLD || blk(x0 + 32 * S - 1) == bd) {
                    uint32_t *chunk = (FOLD ? s_dst[bd] : dst0) + x0;
#pragma unroll
                    for (int k = 0; k < S; ++k) chunk[k * 32 + lane] = r[u][k];
                } else {
#pragma unroll
                    for (int k = 0; k < S; ++k) {
                        const int64_t x = x0 + k * 32 + lane;
                        s_dst[blk(x)][x] = r[u][k];
                    }
                }
            }
        }
    }
    // tail: positions from 32 * groups * S on, element by element
    const int64_t tail0 = static_cast<int64_t>(groups) * 32 * S;
    const int64_t tid = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    const int64_t nthr = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t x = tail0 + tid; x < P.N; x += nthr) {
        const int64_t p = dpinv_pos(P, x);
        if (DIR == ROW_R2C) s_dst[blk(p)][p] = s_src[blk(x)][x];
        else s_dst[blk(x)][x] = s_src[blk(p)][p];
    }
}

template <int S, int DIR, bool FOLD>
__global__ void __launch_bounds__(kRegThreads) skinny_reg_kernel(SkinnyRowParams P) {
    skinny_reg_row<S, DIR, FOLD>(P);
}

// All n long-row shuffles in ONE cooperative launch (P.gbar != nullptr): row i of the rolling
// scheme writes the location row i - 1 (R2C) / row i + 1 (C2R) read and reads nothing another
// row of this launch writes, so the only hazard between consecutive rows is write-after-read,
// closed by a grid barrier: every CTA's loads of row i were consumed by its stores (complete)
// before it arrives; no CTA writes row i + 1's destination before all have arrived.  The
// cooperative launch guarantees the co-residency the barrier needs (or fails cleanly).
template <int S, int DIR, bool FOLD>
__global__ void __launch_bounds__(kRegThreads) skinny_reg_all_kernel(SkinnyRowParams P) {
    const unsigned int nblk = gridDim.x * gridDim.y;
    for (int32_t i = 0; i < P.n; ++i) {
        P.i = i;
        skinny_reg_row<S, DIR, FOLD>(P);
        if (i + 1 == P.n) break;
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(P.gbar, 1u);
            const unsigned int target = static_cast<unsigned int>(i + 1) * nblk;
            unsigned int v;
            while (true) {
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(P.gbar) : "memory");
                if (v >= target) break;
                __nanosleep(64);
            }
        }
        __syncthreads();  // also: the shared tables of row i are rebuilt for row i + 1
    }
}

template <int S, int DIR, bool FOLD>
cudaError_t launch_s(const SkinnyRowParams &P, cudaStream_t st) {
    if (P.gbar) {
        auto kern = skinny_reg_all_kernel<S, DIR, FOLD>;
        const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kRegThreads, 0);
        if (resident < static_cast<int64_t>(P.batch)) {
            // more matrices than co-resident CTAs: one launch per row (stream-ordered)
            SkinnyRowParams Q = P;
            Q.gbar = nullptr;
            for (int32_t i = 0; i < P.n; ++i) {
                Q.i = i;
                const cudaError_t e = launch_s<S, DIR, FOLD>(Q, st);
                if (e != cudaSuccess) return e;
            }
            return cudaSuccess;
        }
        const int64_t warps = (P.N / S + 31) / 32;
        int64_t grid = (warps * 32 + kRegThreads - 1) / kRegThreads;
        const int64_t per = resident / P.batch;  // every CTA of the launch co-resident
        if (grid > per) grid = per;
        if (grid < 1) grid = 1;
        SkinnyRowParams Q = P;
        void *args[] = {&Q};
        return cudaLaunchCooperativeKernel(reinterpret_cast<const void *>(kern),
                                           dim3(static_cast<unsigned>(grid), static_cast<unsigned>(P.batch)),
                                           dim3(kRegThreads), args, 0, st);
    }
    auto kern = skinny_reg_kernel<S, DIR, FOLD>;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kRegThreads, 0);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t warps = (P.N / S + 31) / 32;
    int64_t grid = (warps * 32 + kRegThreads - 1) / kRegThreads;
    const int64_t per = (resident + P.batch - 1) / P.batch;
    if (grid > per) grid = per;
    if (grid < 1) grid = 1;
    kern<<<dim3(static_cast<unsigned>(grid), static_cast<unsigned>(P.batch)), kRegThreads, 0, st>>>(P);
    return cudaGetLastError();
}

template <int S>
cudaError_t launch_d(const SkinnyRowParams &P, int dir, cudaStream_t st) {
    if (dir == ROW_R2C) return P.fold ? launch_s<S, ROW_R2C, true>(P, st) : launch_s<S, ROW_R2C, false>(P, st);
    return P.fold ? launch_s<S, ROW_C2R, true>(P, st) : launch_s<S, ROW_C2R, false>(P, st);
}

template <int S>
cudaError_t dispatch(const SkinnyRowParams &P, int dir, cudaStream_t st) {
    if constexpr (S > 32) {
        return cudaErrorNotSupported;
    } else {
        return P.n == S ? launch_d<S>(P, dir, st) : dispatch<S + 1>(P, dir, st);
    }
}

}  // namespace

cudaError_t launch_skinny_row_reg(const SkinnyRowParams &P, int dir, cudaStream_t st) {
    if (P.n < 2 || P.n > 32) return cudaErrorNotSupported;
    return dispatch<2>(P, dir, st);
}

}  // namespace ipt
