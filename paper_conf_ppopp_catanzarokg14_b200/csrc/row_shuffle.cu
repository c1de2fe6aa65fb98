// Row-shuffle kernel (§3 Eq. 24, §4.2 Eq. 31, §4.5 :751).
//
// Every row of the M x N engine view is permuted independently by the same formula
// (Theorem 3: d'_i is a bijection for every i).  B200 realisation of the paper's
// "on-chip row shuffle" (:751): the whole row is staged in shared memory (the K20c used
// its register file), then each thread gathers the outputs of one 16-byte chunk and
// writes them back with a single vector store.  Global traffic: one read and one write of
// every element, 16-byte aligned vectors in the interior of the row, element accesses in
// the ragged head/tail chunks (rows are 16-byte aligned only when N*eb % 16 == 0).
//
// Gather indices (derived from Eq. 24 by splitting j = l*b + h, l < c, h < b; checked
// against the oracle's Eq. 31 / Eq. 24 by the parity tests):
//   d'_i(l b + h)   = c * ((E_l + (h a mod b)) mod b) + (i + l) mod c
//   E_l             = (floor(i/c) + [l >= c - i mod c] - a [i + l >= M]) mod b
// and its inverse for output position p = col * c + rho:
//   l = (rho - i) mod c,  h = a^{-1} (col - E_l) mod b,  d'^{-1}_i(p) = l b + h,
// where a^{-1} E_l = a^{-1} floor(i/c) + a^{-1} [rho < i mod c] - [i + l >= M]  (mod b).
#include "plan.h"

namespace ipt {

namespace {

constexpr int kRowThreads = 512;

template <int EB>
struct RowGather {
    // Per-row invariants.
    int32_t i, Ri, Qb, Gi, Mi;
    __device__ __forceinline__ void init(const RowParams &P, int32_t row) {
        i = row;
        uint32_t Qi = fdiv(static_cast<uint32_t>(row), P.fd_c);
        Ri = row - static_cast<int32_t>(Qi) * P.c;
        uint32_t Qbm = fmod_(Qi, P.fd_b);
        Qb = static_cast<int32_t>(Qbm);
        Gi = static_cast<int32_t>(mulmod(static_cast<uint32_t>(P.ainv), Qbm, P.fd_b, P.wide));
        Mi = P.M - row;  // [i + l >= M]  <=>  l >= M - i
    }
    // C2R: source column of output position p (Eq. 31).
    __device__ __forceinline__ int32_t c2r(const RowParams &P, int32_t p) const {
        uint32_t col = fdiv(static_cast<uint32_t>(p), P.fd_c);
        int32_t rho = p - static_cast<int32_t>(col) * P.c;
        bool f1 = rho < Ri;
        int32_t l = rho - Ri + (f1 ? P.c : 0);
        int32_t h = static_cast<int32_t>(mulmod(static_cast<uint32_t>(P.ainv), col, P.fd_b, P.wide));
        h += (l >= Mi) ? 1 : 0;
        h -= Gi;
        h += (h < 0) ? P.b : 0;
        h -= (h >= P.b) ? P.b : 0;
        if (f1) {
            h -= P.ainv;
            h += (h < 0) ? P.b : 0;
        }
        return l * P.b + h;
    }
    // R2C: source column of output position j (Eq. 24 used as a gather).
    __device__ __forceinline__ int32_t r2c(const RowParams &P, int32_t j) const {
        uint32_t l = fdiv(static_cast<uint32_t>(j), P.fd_b);
        int32_t h = j - static_cast<int32_t>(l) * P.b;
        int32_t E = Qb + ((static_cast<int32_t>(l) >= P.c - Ri) ? 1 : 0);
        if (static_cast<int32_t>(l) >= Mi) E -= P.amodb;
        E += (E < 0) ? P.b : 0;
        E -= (E >= P.b) ? P.b : 0;
        int32_t ha = static_cast<int32_t>(mulmod(static_cast<uint32_t>(h), static_cast<uint32_t>(P.amodb), P.fd_b, P.wide));
        int32_t col = E + ha;
        col -= (col >= P.b) ? P.b : 0;
        int32_t rho = Ri + static_cast<int32_t>(l);
        rho -= (rho >= P.c) ? P.c : 0;
        return P.c * col + rho;
    }
};

template <int EB, int DIR>
__global__ void __launch_bounds__(kRowThreads) row_shuffle_kernel(RowParams P) {
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
        for (int k = threadIdx.x; k < nch; k += blockDim.x) {
            const int lo = k * 16 - off;
            if (lo >= 0 && lo + 16 <= nbytes) {
                reinterpret_cast<uint4 *>(smem)[k] = ldg16(row0 + 16 * k);
            } else {
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    const int q = lo + e * EB;
                    if (q >= 0 && q < nbytes)
                        reinterpret_cast<T *>(smem + off)[q / EB] = *reinterpret_cast<const T *>(row + q);
                }
            }
        }
        __syncthreads();

        // ---- gather + write back, one 16-byte chunk per thread ----------------------
        RowGather<EB> G;
        G.init(P, i);
        const T *src = reinterpret_cast<const T *>(smem + off);
        for (int k = threadIdx.x; k < nch; k += blockDim.x) {
            const int lo = k * 16 - off;
            const int p0 = lo / EB;  // may be negative in the head chunk
            if (lo >= 0 && lo + 16 <= nbytes) {
                union { uint4 u; T t[PER]; } v;
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    const int32_t s = DIR == ROW_C2R ? G.c2r(P, p0 + e) : G.r2c(P, p0 + e);
                    v.t[e] = src[s];
                }
                stg16(row0 + 16 * k, v.u);
            } else {
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    const int p = p0 + e;
                    if (p >= 0 && p < P.N) {
                        const int32_t s = DIR == ROW_C2R ? G.c2r(P, p) : G.r2c(P, p);
                        reinterpret_cast<T *>(row)[p] = src[s];
                    }
                }
            }
        }
        __syncthreads();  // smem is reused by the next row
    }
}

template <int EB, int DIR>
cudaError_t launch_row_t(const RowParams &P, cudaStream_t st) {
    const size_t smem = row_smem_bytes(P.N, EB);
    auto kern = row_shuffle_kernel<EB, DIR>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
    if (e != cudaSuccess) return e;
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kRowThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    const int64_t rows = static_cast<int64_t>(P.M) * P.batch;
    int64_t grid = static_cast<int64_t>(sms) * per_sm * 4;
    if (grid > rows) grid = rows;
    kern<<<static_cast<unsigned>(grid), kRowThreads, smem, st>>>(P);
    return cudaGetLastError();
}

}  // namespace

size_t row_smem_bytes(int64_t N, int eb) { return static_cast<size_t>(N) * eb + 16; }
int row_block_threads() { return kRowThreads; }

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
