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
#include <algorithm>

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
// Storage locations of row shuffle i's source and destination blocks (plan.h).
__device__ __forceinline__ int32_t sk_src_loc(const SkinnyRowParams &P, int DIR, int32_t rho) {
    int32_t L;
    if (DIR == ROW_R2C) {
        if (P.i == P.n - 1) return P.n;
        L = P.i + 1 + rho;
    } else {
        L = P.i + rho;
    }
    return L >= P.n ? L - P.n : L;
}
__device__ __forceinline__ int32_t sk_dst_loc(const SkinnyRowParams &P, int DIR, int32_t rho) {
    int32_t L;
    if (DIR == ROW_R2C) {
        L = P.i + rho;
    } else {
        if (P.i == 0) return P.n;
        L = P.i - 1 + rho;
    }
    return L >= P.n ? L - P.n : L;
}

template <int EB, int DIR, bool FOLD>
__global__ void __launch_bounds__(kSkThreads) skinny_row_kernel(SkinnyRowParams P) {
    using T = typename Word<EB>::T;
    extern __shared__ __align__(16) unsigned char smem[];
    int64_t *run_lb = reinterpret_cast<int64_t *>(smem);
    int64_t *run_h = run_lb + 32;
    T **src_b = reinterpret_cast<T **>(smem + 512);  // [c] source row base per block
    T **dst_b = src_b + 32;                          // [c] destination row base per block
    T *buf = reinterpret_cast<T *>(smem + 1024);
    const uint32_t sbuf = static_cast<uint32_t>(__cvta_generic_to_shared(buf));
    const int n = P.n;
    const int64_t L = static_cast<int64_t>(n) * P.T;
    // batches: matrix blockIdx.y of the launch, its own tmp row
    char *const Am = P.A + static_cast<int64_t>(blockIdx.y) * P.mat_stride;
    char *const tmpm = P.tmp + static_cast<int64_t>(blockIdx.y) * P.tmp_stride;
    const int lt = 31 - __clz(P.T);  // T is a power of two
    const int nblk = FOLD ? P.c : 1;
    if (threadIdx.x < nblk) {
        const int32_t ls = sk_src_loc(P, DIR, FOLD ? threadIdx.x : 0);
        const int32_t ld = sk_dst_loc(P, DIR, FOLD ? threadIdx.x : 0);
        src_b[threadIdx.x] = reinterpret_cast<T *>(ls == n ? tmpm : Am + ls * P.N * EB);
        dst_b[threadIdx.x] = reinterpret_cast<T *>(ld == n ? tmpm : Am + ld * P.N * EB);
    }
    // Without folding one base serves the whole row (kept in registers).
    const int32_t l0 = sk_src_loc(P, DIR, 0), d0 = sk_dst_loc(P, DIR, 0);
    T *const src0 = reinterpret_cast<T *>(l0 == n ? tmpm : Am + l0 * P.N * EB);
    T *const dst0 = reinterpret_cast<T *>(d0 == n ? tmpm : Am + d0 * P.N * EB);
    auto srcb = [&](int64_t x) -> T * {
        return FOLD ? src_b[fdiv(static_cast<uint32_t>(x), P.fd_b)] : src0;
    };
    auto dstb = [&](int64_t x) -> T * {
        return FOLD ? dst_b[fdiv(static_cast<uint32_t>(x), P.fd_b)] : dst0;
    };

    for (int64_t win = blockIdx.x; win * L < P.N; win += gridDim.x) {
        const int64_t x0 = win * L;
        const int32_t len = static_cast<int32_t>(min(L, P.N - x0));
        // run starts: class r of the window starts at x0 + r; run r lies in block lb / b
        if (threadIdx.x < n) {
            int64_t lb, h;
            dpinv(P, x0 + threadIdx.x, lb, h);
            run_lb[threadIdx.x] = lb;
            run_h[threadIdx.x] = h;
        }
        if (DIR == ROW_R2C) {
            __syncthreads();  // block bases
            // stage the source window, sorted by residue class
            for (int32_t v = threadIdx.x; v < len; v += blockDim.x) {
                const uint32_t t = fdiv(static_cast<uint32_t>(v), P.fd_n);
                const uint32_t r = static_cast<uint32_t>(v) - t * n;
                const int64_t x = x0 + v;
                cp_async_e<EB>(sbuf + (r * P.Tp + t) * EB, srcb(x) + x);
            }
            asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
            __syncthreads();
            // write the n output runs
            for (int32_t e = threadIdx.x; e < n * P.T; e += blockDim.x) {
                const int32_t r = e >> lt, t = e & (P.T - 1);
                if (t * n + r >= len) continue;
                int64_t h = run_h[r] + t;
                if (h >= P.b) h -= P.b;
                const int64_t y = run_lb[r] + h;
                dstb(run_lb[r])[y] = buf[r * P.Tp + t];
            }
        } else {
            __syncthreads();  // run tables, block bases
            // gather the n source runs of the output window
            for (int32_t e = threadIdx.x; e < n * P.T; e += blockDim.x) {
                const int32_t r = e >> lt, t = e & (P.T - 1);
                if (t * n + r >= len) continue;
                int64_t h = run_h[r] + t;
                if (h >= P.b) h -= P.b;
                cp_async_e<EB>(sbuf + (r * P.Tp + t) * EB, srcb(run_lb[r]) + run_lb[r] + h);
            }
            asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
            __syncthreads();
            // write the window
            for (int32_t v = threadIdx.x; v < len; v += blockDim.x) {
                const uint32_t t = fdiv(static_cast<uint32_t>(v), P.fd_n);
                const uint32_t r = static_cast<uint32_t>(v) - t * n;
                const int64_t x = x0 + v;
                dstb(x)[x] = buf[r * P.Tp + t];
            }
        }
        __syncthreads();  // tables and buffer are reused by the next window
    }
}

// Skinny column pass: columns of only n <= 32 elements, so one CTA stages ALL n rows of C
// consecutive columns (n coalesced row segments), then writes out[i][j] = in[sigma_j(i)][j]:
//   ROT       sigma_j(i) = (i + sign floor(j/b)) mod n            (Eq. 23 / Eq. 36)
//   C2R_SHUF  sigma_j(i) = (j + q(i)) mod n                       (Eq. 26 = p_j o q)
//   R2C_SHUF  sigma_j(i) = q^{-1}((i - j) mod n)                  (Eqs. 34-35)
// with the rolling-row remaps of the skinny engine on the input or output side.  A CTA
// reads its columns completely before writing them and CTAs own disjoint columns.
template <int EB, int MODE, bool FOLD>
__global__ void __launch_bounds__(kSkThreads) skinny_col_kernel(SkinnyColParams P) {
    using T = typename Word<EB>::T;
    extern __shared__ __align__(16) unsigned char smem[];
    int32_t *qinv_s = reinterpret_cast<int32_t *>(smem);  // 32 entries
    T *buf = reinterpret_cast<T *>(smem + 128);            // [n][C]
    __shared__ T *rowp_s[32];                              // output row of each logical row
    __shared__ const T *segp_s[32];                        // the block's source segment of each row
    __shared__ bool fast_s[32];                            // ... staged with 16-byte chunks
    const uint32_t sbuf = static_cast<uint32_t>(__cvta_generic_to_shared(buf));
    const int n = P.n, C = P.C;
    const int64_t pitch = P.N;  // in elements
    // batches: matrix blockIdx.y of the launch, its own tmp row
    T *A = reinterpret_cast<T *>(P.A + static_cast<int64_t>(blockIdx.y) * P.mat_stride);
    T *tmp = reinterpret_cast<T *>(P.tmp + static_cast<int64_t>(blockIdx.y) * P.tmp_stride);
    if (threadIdx.x < 32) qinv_s[threadIdx.x] = P.qinv[threadIdx.x];
    for (int64_t j0 = static_cast<int64_t>(blockIdx.x) * C; j0 < P.N; j0 += static_cast<int64_t>(gridDim.x) * C) {
        const int32_t cols = static_cast<int32_t>(min(static_cast<int64_t>(C), P.N - j0));
        // stage: row s of the view (remap -1: stored at s-1, row 0 in tmp)
        // (folded: + floor(j/b) mod n on the rolled side; rho is constant within a block)
        auto row_of = [&](int s, int64_t j) -> const T * {
            if (P.remap >= 0) return A + s * pitch;
            if (s == 0) return tmp;
            int32_t L = s - 1;
            if (FOLD) {
                L += static_cast<int32_t>(fdiv(static_cast<uint32_t>(j), P.fd_b));
                L -= L >= n ? n : 0;
            }
            return A + L * pitch;
        };
        // The block's row segments: source pointer of each row in a shared table (n threads),
        // then every (row, 16-byte chunk) pair of the fast rows in one flattened loop -- the
        // per-row pointer / fold / alignment work is done once per row, not once per thread.
        if (threadIdx.x < n) {
            const int s = threadIdx.x;
            const T *row0 = row_of(s, j0);
            const bool one_base = !FOLD || row_of(s, j0 + cols - 1) == row0;
            const T *seg = row0 + j0;
            segp_s[s] = seg;
            fast_s[s] = one_base && (reinterpret_cast<uintptr_t>(seg) & 15) == 0 && (cols * EB) % 16 == 0;
        }
        __syncthreads();
        const int nch = cols * EB / 16;  // 16-byte chunks (cp.async.cg): 4-byte cp.async runs at ~75 % of this rate
        if (nch > 2 * static_cast<int>(blockDim.x)) {
            // long rows (small n): per row, each thread several chunks
            for (int s = 0; s < n; ++s) {
                if (!fast_s[s]) continue;
                const char *seg = reinterpret_cast<const char *>(segp_s[s]);
                for (int ch = threadIdx.x; ch < nch; ch += blockDim.x)
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;"
                                 :: "r"(sbuf + s * C * EB + ch * 16), "l"(seg + ch * 16) : "memory");
            }
        } else {
            // short rows (large n): every (row, chunk) pair in one flattened loop
            int s = 0, ch = threadIdx.x;
            while (ch >= nch && s < n) {  // (nch < blockDim only for the last, narrow block)
                ch -= nch;
                ++s;
            }
            for (; s < n;) {
                if (fast_s[s])
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;"
                                 :: "r"(sbuf + s * C * EB + ch * 16), "l"(reinterpret_cast<const char *>(segp_s[s]) + ch * 16)
                                 : "memory");
                ch += blockDim.x;
                while (ch >= nch && s < n) {
                    ch -= nch;
                    ++s;
                }
            }
        }
        {
            for (int s2 = 0; s2 < n; ++s2) {  // rows straddling a fold block or misaligned: per element
                if (fast_s[s2]) continue;
                const T *row0 = row_of(s2, j0);
                const bool one_base = !FOLD || row_of(s2, j0 + cols - 1) == row0;
                for (int32_t x = threadIdx.x; x < cols; x += blockDim.x)
                    cp_async_e<EB>(sbuf + (s2 * C + x) * EB, (one_base ? row0 : row_of(s2, j0 + x)) + j0 + x);
            }
        }
        asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
        __syncthreads();
        // Store: thread = column (coalesced per row), rows inner.  The output row of logical
        // row i is the same for every column of the block (the folded rotation amount rho =
        // floor(j/b) is constant within a block unless it straddles a multiple of b), so its
        // pointer comes from a per-block shared table; the source row index steps with i.
        auto out_row = [&](int i, int32_t rho) -> T * {
            if (P.remap <= 0) return A + i * pitch;
            if (i == n - 1) return tmp;
            int32_t L = i + 1 + (FOLD ? rho : 0);
            L -= L >= n ? n : 0;
            return A + L * pitch;
        };
        auto rot_shift = [&](int32_t qd) { return P.rot_sign > 0 ? qd : (qd == 0 ? 0 : n - qd); };
        const int32_t rho0 = (FOLD || MODE == COL_ROT) ? static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0), P.fd_b)) : 0;
        const bool one_rho = !(FOLD || MODE == COL_ROT) ||
                             static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + cols - 1), P.fd_b)) == rho0;
        if (threadIdx.x < n) rowp_s[threadIdx.x] = out_row(threadIdx.x, rho0);
        __syncthreads();
        for (int32_t x = threadIdx.x; x < cols; x += blockDim.x) {
            const int64_t j = j0 + x;  // < N < 2^31
            const int32_t jm = static_cast<int32_t>(fmod_(static_cast<uint32_t>(j), P.fd_n));
            const int32_t rho = one_rho ? rho0 : static_cast<int32_t>(fdiv(static_cast<uint32_t>(j), P.fd_b));
            // source row of output row 0, then +1 (mod n) per row for ROT and R2C
            int32_t s0;
            if (MODE == COL_ROT) s0 = rot_shift(rho);
            else if (MODE == COL_R2C_SHUF) s0 = jm == 0 ? 0 : n - jm;  // u = (0 - jm) mod n
            else s0 = 0;
            const T *col = buf + x;
            for (int i = 0; i < n; ++i) {
                int32_t src;
                if (MODE == COL_ROT) {
                    src = s0;
                } else if (MODE == COL_C2R_SHUF) {
                    src = jm + P.q[i];
                    src -= src >= n ? n : 0;
                } else {
                    src = qinv_s[s0];
                }
                // (plain rows: one multiply-add; rolled rows: the block's table)
                T *orow = P.remap <= 0 ? A + i * pitch : one_rho ? rowp_s[i] : out_row(i, rho);
                orow[j] = col[src * C];
                if (MODE != COL_C2R_SHUF) {
                    ++s0;
                    s0 -= s0 >= n ? n : 0;
                }
            }
        }
        __syncthreads();  // the buffer is refilled by the next column block
    }
}

template <int EB, int MODE>
cudaError_t launch_col_t(const SkinnyColParams &P, cudaStream_t st) {
    const size_t smem = skinny_col_smem(P.n, P.C, EB);
    auto kern = P.fold ? skinny_col_kernel<EB, MODE, true> : skinny_col_kernel<EB, MODE, false>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kSkThreads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t blocks = (P.N + P.C - 1) / P.C;
    const int64_t per = std::max<int64_t>(1, (4 * static_cast<int64_t>(resident) + P.batch - 1) / P.batch);
    const int64_t grid = blocks < per ? blocks : per;  // ~4 waves of CTAs over the whole batch
    kern<<<dim3(static_cast<unsigned>(grid), static_cast<unsigned>(P.batch)), kSkThreads, smem, st>>>(P);
    return cudaGetLastError();
}

template <int EB>
cudaError_t launch_col_e(const SkinnyColParams &P, cudaStream_t st) {
    switch (P.mode) {
        case COL_ROT: return launch_col_t<EB, COL_ROT>(P, st);
        case COL_C2R_SHUF: return launch_col_t<EB, COL_C2R_SHUF>(P, st);
        case COL_R2C_SHUF: return launch_col_t<EB, COL_R2C_SHUF>(P, st);
        default: return cudaErrorInvalidValue;
    }
}

template <int EB, int DIR>
cudaError_t launch_t(const SkinnyRowParams &P, cudaStream_t st) {
    const size_t smem = skinny_row_smem(P.n, P.Tp, EB);
    auto kern = P.fold ? skinny_row_kernel<EB, DIR, true> : skinny_row_kernel<EB, DIR, false>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kSkThreads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t L = static_cast<int64_t>(P.n) * P.T;
    const int64_t wins = (P.N + L - 1) / L;
    const int64_t per = std::max<int64_t>(1, (4 * static_cast<int64_t>(resident) + P.batch - 1) / P.batch);
    const int64_t grid = wins < per ? wins : per;
    kern<<<dim3(static_cast<unsigned>(grid), static_cast<unsigned>(P.batch)), kSkThreads, smem, st>>>(P);
    return cudaGetLastError();
}

}  // namespace

size_t skinny_row_smem(int n, int Tp, int eb) { return 1024 + static_cast<size_t>(n) * Tp * eb; }
size_t skinny_col_smem(int n, int C, int eb) { return 128 + static_cast<size_t>(n) * C * eb; }

cudaError_t launch_skinny_col(const SkinnyColParams &P, int eb, cudaStream_t st) {
    switch (eb) {
        case 4: return launch_col_e<4>(P, st);
        case 8: return launch_col_e<8>(P, st);
        case 16: return launch_col_e<16>(P, st);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_skinny_row(const SkinnyRowParams &P, int dir, int eb, cudaStream_t st) {
    if (P.reg && eb == 4) return launch_skinny_row_reg(P, dir, st);
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
