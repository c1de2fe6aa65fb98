// Skinny long-row shuffle (§6.1 :1039-1047, Fig. 7).
//
// For AoS <-> SoA the array has a tiny dimension n (fields, <= 32) and a huge one N
// (count).  The paper's specialisation "performs all column operations in on-chip memory,
// since we can guarantee that the number of rows is very small by choosing the C2R or R2C
// algorithm appropriately" (:1045): the engine view is n rows of N elements, the column
// passes are n-row tiles (col_tile.cu with one CTA per tile), and the row shuffle runs on
// rows far larger than shared memory.  This file is that row shuffle.
//
// Structure used (derived in DESIGN.md §"Skinny"; checked by the GPU parity tests):
// with q = (x - i) mod N, l = q mod c, h = (a^{-1} floor(q/c) + [i + l >= n]) mod b,
//     d'^{-1}_i(x) = l b + h,
// and x -> x + n leaves l unchanged and adds exactly 1 to h (mod b) because a^{-1} a = 1
// (mod b).  Hence a window of n*T consecutive positions splits into n residue classes mod
// n, each of which is a contiguous run of T positions (cyclic inside segment l) on the
// other side of the permutation:
//   * R2C (AoS -> SoA): out[d'^{-1}_i(k)] = src[k].  A CTA stages a source window
//     [s, s + nT) (coalesced), re-sorted in shared memory by residue class, and writes n
//     contiguous output runs.
//   * C2R (SoA -> AoS): out[j] = src[d'^{-1}_i(j)].  A CTA reads the n contiguous source
//     runs of an output window [w0, w0 + nT) and writes the window (coalesced).
// Every element is read once and written once.  In-place safety comes from the caller:
// the destination row is never the source row (rolling rows + one tmp row, api.cu).
#include "plan.h"

namespace ipt {
namespace {

constexpr int kSkThreads = 256;

template <int EB>
__device__ __forceinline__ void cp_async_e(uint32_t dst, const void *src) {
    if constexpr (EB == 16)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(src) : "memory");
    else
        asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" :: "r"(dst), "l"(src), "n"(EB) : "memory");
}

// d'^{-1}_i(x) = l b + h (closed form above); returns l * b and h separately.
__device__ __forceinline__ void dpinv(const SkinnyRowParams &P, int64_t x, int64_t &lb, int64_t &h) {
    int64_t q = x - P.i;
    if (q < 0) q += P.N;
    const int64_t l = q % P.c;
    h = (P.ainv * (q / P.c)) % P.b;  // a^{-1} < b, floor(q/c) < b, b < 2^31: fits in 64 bits
    if (P.i + l >= P.n) h = h + 1 == P.b ? 0 : h + 1;
    lb = l * P.b;
}

// Shared memory: run tables [n] x (l*b, h) as int64, then the window re-sorted by residue
// class: element t of class r at row r, column t (row pitch Tp elements).
template <int EB, int DIR>
__global__ void __launch_bounds__(kSkThreads) skinny_row_kernel(SkinnyRowParams P) {
    using T = typename Word<EB>::T;
    extern __shared__ __align__(16) unsigned char smem[];
    int64_t *run_lb = reinterpret_cast<int64_t *>(smem);
    int64_t *run_h = run_lb + 32;
    T *buf = reinterpret_cast<T *>(smem + 512);
    const uint32_t sbuf = static_cast<uint32_t>(__cvta_generic_to_shared(buf));
    const int n = P.n;
    const int64_t L = static_cast<int64_t>(n) * P.T;
    const int lt = 31 - __clz(P.T);  // T is a power of two
    const T *src = reinterpret_cast<const T *>(P.src);
    T *dst = reinterpret_cast<T *>(P.dst);

    for (int64_t win = blockIdx.x; win * L < P.N; win += gridDim.x) {
        const int64_t x0 = win * L;
        const int32_t len = static_cast<int32_t>(min(L, P.N - x0));
        // run starts: class r of the window starts at x0 + r
        if (threadIdx.x < n) {
            int64_t lb, h;
            dpinv(P, x0 + threadIdx.x, lb, h);
            run_lb[threadIdx.x] = lb;
            run_h[threadIdx.x] = h;
        }
        if (DIR == ROW_R2C) {
            // stage the source window, sorted by residue class
            for (int32_t v = threadIdx.x; v < len; v += blockDim.x) {
                const uint32_t t = fdiv(static_cast<uint32_t>(v), P.fd_n);
                const uint32_t r = static_cast<uint32_t>(v) - t * n;
                cp_async_e<EB>(sbuf + (r * P.Tp + t) * EB, src + x0 + v);
            }
            asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
            __syncthreads();
            // write the n output runs
            for (int32_t e = threadIdx.x; e < n * P.T; e += blockDim.x) {
                const int32_t r = e >> lt, t = e & (P.T - 1);
                if (t * n + r >= len) continue;
                int64_t h = run_h[r] + t;
                if (h >= P.b) h -= P.b;
                dst[run_lb[r] + h] = buf[r * P.Tp + t];
            }
        } else {
            __syncthreads();  // run tables
            // gather the n source runs of the output window
            for (int32_t e = threadIdx.x; e < n * P.T; e += blockDim.x) {
                const int32_t r = e >> lt, t = e & (P.T - 1);
                if (t * n + r >= len) continue;
                int64_t h = run_h[r] + t;
                if (h >= P.b) h -= P.b;
                cp_async_e<EB>(sbuf + (r * P.Tp + t) * EB, src + run_lb[r] + h);
            }
            asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
            __syncthreads();
            // write the window
            for (int32_t v = threadIdx.x; v < len; v += blockDim.x) {
                const uint32_t t = fdiv(static_cast<uint32_t>(v), P.fd_n);
                const uint32_t r = static_cast<uint32_t>(v) - t * n;
                dst[x0 + v] = buf[r * P.Tp + t];
            }
        }
        __syncthreads();  // tables and buffer are reused by the next window
    }
}

template <int EB, int DIR>
cudaError_t launch_t(const SkinnyRowParams &P, cudaStream_t st) {
    const size_t smem = skinny_row_smem(P.n, P.Tp, EB);
    auto kern = skinny_row_kernel<EB, DIR>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kSkThreads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t L = static_cast<int64_t>(P.n) * P.T;
    const int64_t wins = (P.N + L - 1) / L;
    const int64_t grid = wins < 4 * static_cast<int64_t>(resident) ? wins : 4 * static_cast<int64_t>(resident);
    kern<<<static_cast<unsigned>(grid), kSkThreads, smem, st>>>(P);
    return cudaGetLastError();
}

}  // namespace

size_t skinny_row_smem(int n, int Tp, int eb) { return 512 + static_cast<size_t>(n) * Tp * eb; }

cudaError_t launch_skinny_row(const SkinnyRowParams &P, int dir, int eb, cudaStream_t st) {
    switch (eb * 2 + dir) {
        case 4 * 2 + ROW_C2R: return launch_t<4, ROW_C2R>(P, st);
        case 4 * 2 + ROW_R2C: return launch_t<4, ROW_R2C>(P, st);
        case 8 * 2 + ROW_C2R: return launch_t<8, ROW_C2R>(P, st);
        case 8 * 2 + ROW_R2C: return launch_t<8, ROW_R2C>(P, st);
        case 16 * 2 + ROW_C2R: return launch_t<16, ROW_C2R>(P, st);
        case 16 * 2 + ROW_R2C: return launch_t<16, ROW_R2C>(P, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace ipt
