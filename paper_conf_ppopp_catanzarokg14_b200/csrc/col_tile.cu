// Column-tile kernel (§3 Eqs. 23, 26, §4.1-4.3,
// §4.6-4.7).
//
// A column operation permutes every column independently.  The B200 realisation stages a
// whole column tile -- all M rows x W adjacent columns (W * eb bytes wide) -- on chip,
// spread over the shared memory of a thread-block cluster of K CTAs (each CTA holds a
// band of B = ceil(M/K) rows plus a halo), and makes the operation a single read + write
// pass.  In-place safety: every CTA finishes reading its part of the tile before ANY CTA
// of the cluster writes (cluster barrier with release/acquire); tiles are disjoint byte
// ranges owned by exactly one cluster.  This replaces the paper's multi-pass
// cache-aware rotate (coarse cycle following + fine on-chip rotation, §4.6) and cycle-
// following row permute (§4.7) -- prior art for a K20c without clusters.
//
// Tile-local forms (w = j - j0 is the column inside the tile [j0, j0 + W)):
//  * COL_ROT, gather rotation rho_j = sign * floor(j/b) (Eq. 23 for sign = +1 as the C2R
//    pre-rotation, Eq. 36 for sign = -1 as the R2C post-rotation):
//        out[i][w] = in[(i + rho_{j0+w}) mod M][w]
//    The CTA writing band [r0, r1) reads rows [r0 + min rho, r1 + max rho) -- a contiguous
//    cyclic range (rho varies by < W inside a tile, :767-773 residual bound).
//  * COL_C2R_SHUF, s'_j(i) = (j + q(i)) mod M (Eq. 26 = p_j o q, Eqs. 32-33):
//        out[i][w] = in[(k + w) mod M][w],  k = (j0 + q(i)) mod M.
//    Scatter form: the CTA reads rows [r0, r1 + W - 1) (band + halo, contiguous), builds
//    the skewed row T_k[w] = in[k + w][w] for each k of its band and writes it to output
//    row i = q^{-1}((k - j0) mod M) (Eq. 34).
//  * COL_R2C_SHUF, (s')^{-1}_j(i) = q^{-1}((i - j) mod M) (Eqs. 34-35):
//        out[i][w] = in[q^{-1}((i - w - j0) mod M)][w].
//    The CTA writing band [r0, r1) reads the rows q^{-1}((u - j0) mod M) for
//    u in [r0 - W + 1, r1) (scattered whole sub-rows) and writes its band contiguously.
#include "plan.h"

namespace ipt {

namespace {

constexpr int kColThreads = 512;

// q^{-1}(i) = (floor((c-1+i)/c) b^{-1}) mod a + (((c-1) i) mod c) a  (Eq. 34).
__device__ __forceinline__ int32_t qinv_of(const ColParams &P, int32_t i) {
    uint32_t t = fdiv(static_cast<uint32_t>(P.c - 1 + i), P.fd_c);
    if (t >= static_cast<uint32_t>(P.a)) t -= P.a;  // t <= a
    uint32_t u = mulmod(t, static_cast<uint32_t>(P.binv), P.fd_a, P.wide_a);
    uint32_t im = static_cast<uint32_t>(i) - fdiv(static_cast<uint32_t>(i), P.fd_c) * P.c;
    uint32_t cm = im == 0 ? 0u : static_cast<uint32_t>(P.c) - im;  // ((c-1) i) mod c = (-i) mod c
    return static_cast<int32_t>(u + cm * static_cast<uint32_t>(P.a));
}

__device__ __forceinline__ int32_t mod_M(int64_t v, int32_t M) {
    v %= M;
    return static_cast<int32_t>(v < 0 ? v + M : v);
}

template <int EB, int MODE>
__global__ void __launch_bounds__(kColThreads) col_tile_kernel(ColParams P) {
    using T = typename Word<EB>::T;
    extern __shared__ __align__(16) unsigned char smem[];

    const int32_t W = P.W, lw = P.log2W;
    const int64_t cid = blockIdx.x / P.K;  // cluster id
    const int32_t r = blockIdx.x - static_cast<int32_t>(cid * P.K);
    const int32_t tile = static_cast<int32_t>(cid % P.ntiles);
    const int64_t mat = cid / P.ntiles;
    char *A = P.base + mat * P.mat_stride_bytes;
    const int32_t j0 = tile * W;
    const int32_t Wt = min(W, P.N - j0);
    const int32_t r0 = r * P.B;
    const int32_t r1 = min(P.M, r0 + P.B);
    const int32_t nrows = max(0, r1 - r0);

    // Band geometry per mode.
    int32_t ext, base_off = 0;
    int32_t lo_q = 0, hi_q = 0;
    if (MODE == COL_ROT) {
        lo_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0), P.fd_b));
        hi_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + Wt - 1), P.fd_b));
        // Columns j < b rotate by 0 (Eq. 23): a tile made only of them is left alone.  The
        // whole cluster shares the tile, so the early exit is cluster-uniform.
        if (hi_q == 0) return;
        ext = hi_q - lo_q;
        base_off = P.rot_sign > 0 ? lo_q : -hi_q;  // smallest rotation amount in the tile
    } else {
        ext = W - 1;
    }
    const int32_t nslots = nrows > 0 ? nrows + ext : 0;

    T *slot = reinterpret_cast<T *>(smem);                                       // [nslots][W]
    int32_t *ridx = reinterpret_cast<int32_t *>(smem + static_cast<size_t>(nslots) * W * EB);  // [nslots]

    // ---- phase 1: which global row feeds each slot (C2R: also the destination rows) --
    for (int32_t t = threadIdx.x; t < nslots; t += blockDim.x) {
        int32_t row;
        if (MODE == COL_ROT) {
            row = mod_M(static_cast<int64_t>(r0) + base_off + t, P.M);
        } else if (MODE == COL_C2R_SHUF) {
            row = mod_M(static_cast<int64_t>(r0) + t, P.M);
        } else {
            const int64_t u = static_cast<int64_t>(r0) - (W - 1) + t;
            row = qinv_of(P, mod_M(u - j0, P.M));
        }
        ridx[t] = row;
    }
    __syncthreads();

    // ---- phase 2: load the (skewed) band of the tile into shared memory ------------
    const int32_t nel = nslots << lw;
    for (int32_t e = threadIdx.x; e < nel; e += blockDim.x) {
        const int32_t t = e >> lw, w = e & (W - 1);
        if (w < Wt) {
            const T *g = reinterpret_cast<const T *>(A) + static_cast<int64_t>(ridx[t]) * P.N + j0 + w;
            slot[e] = *g;
        }
    }

    // In-place hazard barrier: the whole tile has been read before anyone writes it.
    if (P.K > 1) cluster_barrier(); else __syncthreads();

    // ---- phase 3: destination rows of the C2R scatter form -----------------------------
    if (MODE == COL_C2R_SHUF) {
        // reuse ridx[0..nrows) for destinations (ridx for sources is no longer needed)
        for (int32_t kk = threadIdx.x; kk < nrows; kk += blockDim.x)
            ridx[kk] = qinv_of(P, mod_M(static_cast<int64_t>(r0) + kk - j0, P.M));
        __syncthreads();
    }

    // ---- phase 4: write ----------------------------------------------------------------
    const int32_t nout = nrows << lw;
    for (int32_t e = threadIdx.x; e < nout; e += blockDim.x) {
        const int32_t kk = e >> lw, w = e & (W - 1);
        if (w >= Wt) continue;
        T v;
        int64_t orow;
        if (MODE == COL_ROT) {
            const int32_t qw = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + w), P.fd_b));
            const int32_t dw = P.rot_sign > 0 ? qw - lo_q : hi_q - qw;  // rho_w - min rho
            v = slot[((kk + dw) << lw) + w];
            orow = r0 + kk;
        } else if (MODE == COL_C2R_SHUF) {
            v = slot[((kk + w) << lw) + w];
            orow = ridx[kk];
        } else {
            v = slot[((kk - w + W - 1) << lw) + w];
            orow = r0 + kk;
        }
        reinterpret_cast<T *>(A)[orow * P.N + j0 + w] = v;
    }
}

template <int EB, int MODE>
void *col_kernel_ptr() {
    return reinterpret_cast<void *>(col_tile_kernel<EB, MODE>);
}

void *col_kernel(int mode, int eb) {
    switch (eb * 4 + mode) {
        case 4 * 4 + COL_ROT: return col_kernel_ptr<4, COL_ROT>();
        case 4 * 4 + COL_C2R_SHUF: return col_kernel_ptr<4, COL_C2R_SHUF>();
        case 4 * 4 + COL_R2C_SHUF: return col_kernel_ptr<4, COL_R2C_SHUF>();
        case 8 * 4 + COL_ROT: return col_kernel_ptr<8, COL_ROT>();
        case 8 * 4 + COL_C2R_SHUF: return col_kernel_ptr<8, COL_C2R_SHUF>();
        case 8 * 4 + COL_R2C_SHUF: return col_kernel_ptr<8, COL_R2C_SHUF>();
        case 16 * 4 + COL_ROT: return col_kernel_ptr<16, COL_ROT>();
        case 16 * 4 + COL_C2R_SHUF: return col_kernel_ptr<16, COL_C2R_SHUF>();
        case 16 * 4 + COL_R2C_SHUF: return col_kernel_ptr<16, COL_R2C_SHUF>();
        default: return nullptr;
    }
}

cudaError_t prepare(void *kern, int K, size_t smem) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
    if (e != cudaSuccess) return e;
    if (K > 8) {
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

}  // namespace

size_t col_smem_bytes(int64_t B, int64_t W, int eb) {
    const int64_t nslots = B + W - 1;
    return static_cast<size_t>(nslots * W * eb + nslots * 4);
}

int col_block_threads() { return kColThreads; }

int col_max_active_clusters(int mode, int eb, int K, size_t smem) {
    void *kern = col_kernel(mode, eb);
    if (!kern || prepare(kern, K, smem) != cudaSuccess) return 0;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    cfg.gridDim = dim3(static_cast<unsigned>(K) * 64);
    cfg.blockDim = dim3(kColThreads);
    cfg.dynamicSmemBytes = smem;
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = K;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, kern, &cfg) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return n;
}

cudaError_t launch_col(const ColParams &P, int mode, int eb, cudaStream_t st, size_t smem) {
    void *kern = col_kernel(mode, eb);
    if (!kern) return cudaErrorInvalidValue;
    cudaError_t e = prepare(kern, P.K, smem);
    if (e != cudaSuccess) return e;
    const int64_t grid = static_cast<int64_t>(P.K) * P.ntiles * P.batch;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    cfg.gridDim = dim3(static_cast<unsigned>(grid));
    cfg.blockDim = dim3(kColThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = P.K;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    void *args[] = {const_cast<ColParams *>(&P)};
    return cudaLaunchKernelExC(&cfg, kern, args);
}

}  // namespace ipt
