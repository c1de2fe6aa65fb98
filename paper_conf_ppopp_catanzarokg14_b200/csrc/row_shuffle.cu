// Row-shuffle kernel (§3 Eq. 24, §4.2 Eq. 31, §4.5 :751).
//
// Every row of the M x N engine view is permuted independently by the same formula
// (Theorem 3: d'_i is a bijection for every i).  B200 realisation of the paper's
// "on-chip row shuffle" (:751): the whole row is staged in shared memory with cp.async
// (16-byte LDGSTS for the aligned interior, element copies for the ragged head/tail --
// rows are 16-byte aligned only when N*eb % 16 == 0), then each thread gathers the
// outputs of one 16-byte chunk from shared memory and writes them back with one vector
// store.  Global traffic: one read and one write of every element.
//
// Gather indices (derived from Eq. 24 by splitting j = l*b + h, l < c, h < b; the parity
// tests check them against the oracle's Eq. 31 / Eq. 24):
//   d'_i(l b + h)   = c * ((E_l + (h a mod b)) mod b) + (i + l) mod c
//   E_l             = (floor(i/c) + [l >= c - i mod c] - a [i + l >= M]) mod b
// and its inverse for output position p = col * c + rho:
//   l = (rho - i) mod c,  h = a^{-1} (col - E_l) mod b,  d'^{-1}_i(p) = l b + h,
// where a^{-1} E_l = a^{-1} floor(i/c) + a^{-1} [rho < i mod c] - [i + l >= M]  (mod b).
// Along consecutive outputs both are evaluated incrementally (§4.4's strength reduction
// taken one step further): one strength-reduced division per 16-byte chunk, then adds
// and compares.
#include "plan.h"

namespace ipt {

namespace {

constexpr int kRowThreadsMax = 512;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
template <int B>
__device__ __forceinline__ void cp_async(uint32_t dst, const void *src) {
    if constexpr (B == 16) {
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(src) : "memory");
    } else {
        asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" :: "r"(dst), "l"(src), "n"(B) : "memory");
    }
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
}

struct RowConst {
    int32_t Ri, Qb, Gi, Mi;
    __device__ __forceinline__ RowConst(const RowParams &P, int32_t i) {
        const uint32_t Qi = fdiv(static_cast<uint32_t>(i), P.fd_c);
        Ri = i - static_cast<int32_t>(Qi) * P.c;
        const uint32_t Qbm = fmod_(Qi, P.fd_b);
        Qb = static_cast<int32_t>(Qbm);
        Gi = static_cast<int32_t>(mulmod(static_cast<uint32_t>(P.ainv), Qbm, P.fd_b, P.wide));
        Mi = P.M - i;  // [i + l >= M]  <=>  l >= M - i
    }
};

// C2R: source of output position p, d'^{-1}_i(p) (Eq. 31), walked along p.
struct C2RIter {
    int32_t rho, l, H;
    __device__ __forceinline__ C2RIter(const RowParams &P, const RowConst &R, int32_t p) {
        const uint32_t col = fdiv(static_cast<uint32_t>(p), P.fd_c);
        rho = p - static_cast<int32_t>(col) * P.c;
        l = rho - R.Ri;
        l += l < 0 ? P.c : 0;
        H = static_cast<int32_t>(mulmod(static_cast<uint32_t>(P.ainv), col, P.fd_b, P.wide));
    }
    __device__ __forceinline__ int32_t src(const RowParams &P, const RowConst &R) const {
        int32_t h = H + (l >= R.Mi ? 1 : 0) - R.Gi;
        h += h < 0 ? P.b : 0;
        h -= h >= P.b ? P.b : 0;
        if (rho < R.Ri) {
            h -= P.ainv;
            h += h < 0 ? P.b : 0;
        }
        return l * P.b + h;
    }
    __device__ __forceinline__ void next(const RowParams &P) {
        ++rho;
        ++l;
        l = l == P.c ? 0 : l;
        if (rho == P.c) {
            rho = 0;
            H += P.ainv;
            H -= H >= P.b ? P.b : 0;
        }
    }
};

// R2C: source of output position j, d'_i(j) (Eq. 24 used as a gather, §4.3 :717).
struct R2CIter {
    int32_t l, h, ha, E, rl;
    __device__ __forceinline__ int32_t E_of(const RowParams &P, const RowConst &R, int32_t ll) const {
        int32_t e = R.Qb + (ll >= P.c - R.Ri ? 1 : 0) - (ll >= R.Mi ? P.amodb : 0);
        e += e < 0 ? P.b : 0;
        e -= e >= P.b ? P.b : 0;
        return e;
    }
    __device__ __forceinline__ R2CIter(const RowParams &P, const RowConst &R, int32_t j) {
        l = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j), P.fd_b));
        h = j - l * P.b;
        ha = static_cast<int32_t>(mulmod(static_cast<uint32_t>(h), static_cast<uint32_t>(P.amodb), P.fd_b, P.wide));
        E = E_of(P, R, l);
        rl = R.Ri + l;
        rl -= rl >= P.c ? P.c : 0;
    }
    __device__ __forceinline__ int32_t src(const RowParams &P, const RowConst &) const {
        int32_t col = E + ha;
        col -= col >= P.b ? P.b : 0;
        return P.c * col + rl;
    }
    __device__ __forceinline__ void next(const RowParams &P, const RowConst &R) {
        ++h;
        ha += P.amodb;
        ha -= ha >= P.b ? P.b : 0;
        if (h == P.b) {
            h = 0;
            ha = 0;
            ++l;
            E = E_of(P, R, l);
            ++rl;
            rl = rl == P.c ? 0 : rl;
        }
    }
};

template <int EB, int DIR>
__global__ void __launch_bounds__(kRowThreadsMax) row_shuffle_kernel(RowParams P) {
    using T = typename Word<EB>::T;
    extern __shared__ __align__(16) unsigned char smem[];
    constexpr int PER = 16 / EB;  // elements per 16-byte chunk
    const int64_t rows_total = static_cast<int64_t>(P.M) * P.batch;
    const int32_t nbytes = P.N * EB;

    for (int64_t r = blockIdx.x; r < rows_total; r += gridDim.x) {
        const int64_t mat = r / P.M;
        const int32_t i = static_cast<int32_t>(r - mat * P.M);
        char *row = P.base + mat * P.mat_stride_bytes + static_cast<int64_t>(i) * nbytes;
        const int off = static_cast<int>(reinterpret_cast<uintptr_t>(row) & 15);  // multiple of EB
        char *row0 = row - off;
        const int nch = (off + nbytes + 15) >> 4;

        // ---- stage the row: smem byte (off + k) holds row byte k --------------------
        const uint32_t sbase = smem_u32(smem);
        for (int k = threadIdx.x; k < nch; k += blockDim.x) {
            const int lo = k * 16 - off;
            if (lo >= 0 && lo + 16 <= nbytes) {
                cp_async<16>(sbase + 16 * k, row0 + 16 * k);
            } else {
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    const int q = lo + e * EB;
                    if (q >= 0 && q < nbytes) cp_async<EB>(sbase + off + q, row + q);
                }
            }
        }
        cp_async_wait_all();
        __syncthreads();

        // ---- gather + write back, one 16-byte chunk per thread ----------------------
        const RowConst R(P, i);
        const T *src = reinterpret_cast<const T *>(smem + off);
        for (int k = threadIdx.x; k < nch; k += blockDim.x) {
            const int lo = k * 16 - off;
            const int p0 = lo / EB;  // negative in a misaligned head chunk
            const int pb = p0 < 0 ? 0 : p0;
            if (lo >= 0 && lo + 16 <= nbytes) {
                union { uint4 u; T t[PER]; } v;
                if (DIR == ROW_C2R) {
                    C2RIter it(P, R, pb);
#pragma unroll
                    for (int e = 0; e < PER; ++e) {
                        v.t[e] = src[it.src(P, R)];
                        if (e + 1 < PER) it.next(P);
                    }
                } else {
                    R2CIter it(P, R, pb);
#pragma unroll
                    for (int e = 0; e < PER; ++e) {
                        v.t[e] = src[it.src(P, R)];
                        if (e + 1 < PER) it.next(P, R);
                    }
                }
                stg16(row0 + 16 * k, v.u);
            } else {
                const int pe = min(p0 + PER, P.N);
                if (DIR == ROW_C2R) {
                    C2RIter it(P, R, pb);
                    for (int p = pb; p < pe; ++p) {
                        reinterpret_cast<T *>(row)[p] = src[it.src(P, R)];
                        it.next(P);
                    }
                } else {
                    R2CIter it(P, R, pb);
                    for (int p = pb; p < pe; ++p) {
                        reinterpret_cast<T *>(row)[p] = src[it.src(P, R)];
                        it.next(P, R);
                    }
                }
            }
        }
        __syncthreads();  // smem is reused by the next row
    }
}

int row_threads(int64_t N, int eb) { return N * eb >= 48 * 1024 ? 512 : 256; }

template <int EB, int DIR>
cudaError_t launch_row_t(const RowParams &P, cudaStream_t st) {
    const size_t smem = row_smem_bytes(P.N, EB);
    const int threads = row_threads(P.N, EB);
    auto kern = row_shuffle_kernel<EB, DIR>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int per_sm_sms = cached_resident_blocks(reinterpret_cast<const void *>(kern), threads, smem);
    if (per_sm_sms < 1) return cudaErrorInvalidConfiguration;
    const int64_t rows = static_cast<int64_t>(P.M) * P.batch;
    int64_t grid = per_sm_sms;
    if (grid > rows) grid = rows;
    kern<<<static_cast<unsigned>(grid), threads, smem, st>>>(P);
    return cudaGetLastError();
}

}  // namespace

size_t row_smem_bytes(int64_t N, int eb) { return static_cast<size_t>(N) * eb + 16; }
int row_block_threads() { return kRowThreadsMax; }

cudaError_t launch_row(const RowParams &P, int dir, int eb, cudaStream_t st) {
    switch (eb * 2 + dir) {
        case 4 * 2 + ROW_C2R: return launch_row_t<4, ROW_C2R>(P, st);
        case 4 * 2 + ROW_R2C: return launch_row_t<4, ROW_R2C>(P, st);
        case 8 * 2 + ROW_C2R: return launch_row_t<8, ROW_C2R>(P, st);
        case 8 * 2 + ROW_R2C: return launch_row_t<8, ROW_R2C>(P, st);
        case 16 * 2 + ROW_C2R: return launch_row_t<16, ROW_C2R>(P, st);
        case 16 * 2 + ROW_R2C: return launch_row_t<16, ROW_R2C>(P, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace ipt
