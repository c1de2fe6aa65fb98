// Column-tile kernel (§3 Eqs. 23, 26, §4.1-4.3,
// §4.6-4.7).
//
// A column operation permutes every column independently.  The B200 realisation stages a
// whole column tile -- all M rows x W adjacent columns (TWB = W * eb bytes wide) -- on
// chip, spread over the shared memory of a GROUP of G CTAs (member r holds the band of
// B rows [r B, r B + B) plus a halo), and makes the operation a single read + write
// pass.  In-place safety: every member finishes reading its part of the tile before ANY
// member writes (a per-group barrier in global memory: release-add on a counter, acquire
// spin until all G members arrived); tiles are disjoint byte ranges owned by exactly one
// group.  This replaces the paper's multi-pass cache-aware rotate (coarse cycle following
// + fine on-chip rotation, §4.6) and cycle-following row permute (§4.7) -- prior art for
// a K20c.
//
// Why software groups rather than hardware clusters: the strided tile access reaches
// copy bandwidth only when each CTA stages a small band (16-64 KB, several CTAs per SM in
// different phases; tools/pattern_probe.cu, profiles/), which needs groups far larger
// than the 16-CTA cluster limit (a 17226-row tile of 128 B is ~2.6 MB).  The kernel is
// persistent and launched cooperatively (every CTA co-resident, so the spin cannot
// deadlock); group g walks the tiles g, g + ngroups, ...
//
// Tile-local forms (w = j - j0 is the column inside the tile [j0, j0 + W)):
//  * COL_ROT, gather rotation rho_j = sign * floor(j/b) (Eq. 23 for sign = +1 as the C2R
//    pre-rotation, Eq. 36 for sign = -1 as the R2C post-rotation):
//        out[i][w] = in[(i + rho_{j0+w}) mod M][w]
//    The member writing band [r0, r1) reads rows [r0 + min rho, r1 + max rho) -- a
//    contiguous cyclic range (rho varies by < W inside a tile, :767-773 residual bound).
//  * COL_C2R_SHUF, s'_j(i) = (j + q(i)) mod M (Eq. 26 = p_j o q, Eqs. 32-33):
//        out[i][w] = in[(k + w) mod M][w],  k = (j0 + q(i)) mod M.
//    Scatter form: the member reads rows [r0, r1 + W - 1) (band + halo, contiguous),
//    builds the skewed row T_k[w] = in[k + w][w] for each k of its band and writes it to
//    output row i = q^{-1}((k - j0) mod M) (Eq. 34).
//  * COL_R2C_SHUF, (s')^{-1}_j(i) = q^{-1}((i - j) mod M) (Eqs. 34-35):
//        out[i][w] = in[q^{-1}((i - w - j0) mod M)][w].
//    The member writing band [r0, r1) reads the rows q^{-1}((u - j0) mod M) for
//    u in [r0 - W + 1, r1) (scattered whole sub-rows) and writes its band contiguously.
//
// Memory access: each staged row is fetched as its 16-byte-aligned hull (TWB/16 + 1
// chunks) with cp.async (LDGSTS, global -> shared without a register round trip), so a
// CTA has its whole band in flight at once; rows are 16-byte aligned only when
// N*eb % 16 == 0, and the hull's extra bytes (neighbouring tiles of the same row) are
// never used.  Chunks that would leave the matrix (row 0 head, row M-1 tail) are fetched
// element by element.  Stores are element-wise (eb bytes per thread, a warp covers
// 32*eb/TWB whole tile rows).
#include "plan.h"

namespace ipt {

namespace {

constexpr int kColThreads = 256;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const void *src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(src) : "memory");
}
template <int B>
__device__ __forceinline__ void cp_async_small(uint32_t dst, const void *src) {
    if constexpr (B == 16) {
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(src) : "memory");
    } else {
        asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" :: "r"(dst), "l"(src), "n"(B) : "memory");
    }
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
}

// q^{-1}(i) = (floor((c-1+i)/c) b^{-1}) mod a + (((c-1) i) mod c) a  (Eq. 34).
__device__ __forceinline__ int32_t qinv_of(const ColParams &P, int32_t i) {
    uint32_t t = fdiv(static_cast<uint32_t>(P.c - 1 + i), P.fd_c);
    if (t >= static_cast<uint32_t>(P.a)) t -= P.a;  // t <= a
    uint32_t u = mulmod(t, static_cast<uint32_t>(P.binv), P.fd_a, P.wide_a);
    uint32_t im = static_cast<uint32_t>(i) - fdiv(static_cast<uint32_t>(i), P.fd_c) * P.c;
    uint32_t cm = im == 0 ? 0u : static_cast<uint32_t>(P.c) - im;  // ((c-1) i) mod c = (-i) mod c
    return static_cast<int32_t>(u + cm * static_cast<uint32_t>(P.a));
}

// v mod M for v >= -kshift*M (kshift = 2 + W/M covers every caller; M < 2^29).
__device__ __forceinline__ int32_t mod_M(int32_t v, uint32_t kshiftM, const FastDiv &fdM) {
    return static_cast<int32_t>(fmod_(static_cast<uint32_t>(v) + kshiftM, fdM));
}

// Group barrier in global memory: counter ctr counts arrivals of all tiles so far.
__device__ __forceinline__ void group_barrier(unsigned int *ctr, unsigned int target) {
    __syncthreads();  // every thread's cp.async data has landed in shared memory
    if (threadIdx.x == 0) {
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
        unsigned int v;
        while (true) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
            if (v >= target) break;
            __nanosleep(64);
        }
    }
    __syncthreads();
}

template <int TWB>
struct TileGeom {
    static constexpr int SLOT = TWB + 16;  // hull bytes per staged row
    static constexpr int CH = TWB / 16 + 1;  // hull chunks per staged row
};

template <int EB, int MODE, int TWB>
__global__ void __launch_bounds__(kColThreads) col_tile_kernel(ColParams P) {
    using T = typename Word<EB>::T;
    constexpr int W = TWB / EB;
    constexpr int LW = W == 1 ? 0 : W == 2 ? 1 : W == 4 ? 2 : W == 8 ? 3 : W == 16 ? 4 : 5;
    constexpr int SLOT = TileGeom<TWB>::SLOT;
    constexpr int CH = TileGeom<TWB>::CH;
    extern __shared__ __align__(16) unsigned char smem[];

    const int32_t g = blockIdx.x / P.G;          // group
    const int32_t r = blockIdx.x - g * P.G;      // member = band index
    if (g >= P.ngroups) return;
    unsigned int *ctr = P.ctr + g;
    const int32_t r0 = r * P.B;
    const int32_t r1 = min(P.M, r0 + P.B);
    const int32_t nrows = max(0, r1 - r0);
    const uint32_t kshM = static_cast<uint32_t>(2 + W / P.M) * static_cast<uint32_t>(P.M);
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    const bool use_barrier = P.G > 1 && !(MODE == COL_COPY && P.rot_sign == 0);
    unsigned int nbar = 0;

    for (int64_t tt = g; tt < P.total_tiles; tt += P.ngroups) {
        const int32_t tile = static_cast<int32_t>(tt % P.ntiles);
        const int64_t mat = tt / P.ntiles;
        char *A = P.base + mat * P.mat_stride_bytes;
        const char *Aend = A + static_cast<int64_t>(P.M) * pitch;
        const int32_t j0 = tile * W;
        const int32_t Wt = min(W, P.N - j0);
        const int32_t j0m = static_cast<int32_t>(fmod_(static_cast<uint32_t>(j0), P.fd_M));

        int32_t ext, base_off = 0, lo_q = 0, hi_q = 0;
        if (MODE == COL_ROT) {
            lo_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0), P.fd_b));
            hi_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + Wt - 1), P.fd_b));
            // Columns j < b rotate by 0 (Eq. 23): a tile made only of them is left alone.
            // Every member sees the same tile, so the skip is group-uniform.
            if (hi_q == 0) continue;
            ext = hi_q - lo_q;
            base_off = P.rot_sign > 0 ? lo_q : -hi_q;  // smallest rotation amount in the tile
        } else if (MODE == COL_COPY) {
            ext = 0;
        } else {
            ext = W - 1;
        }
        const int32_t nslots = nrows > 0 ? nrows + ext : 0;

        unsigned char *stage = smem;                                  // [nslots][SLOT]
        uint8_t *dlt = smem + static_cast<size_t>(nslots) * SLOT;    // [nslots] hull offsets
        int32_t *ridx = reinterpret_cast<int32_t *>(smem + ((static_cast<size_t>(nslots) * (SLOT + 1) + 3) & ~size_t(3)));

        // ---- R2C: the scattered source rows of every slot -----------------------------
        if (MODE == COL_R2C_SHUF) {
            for (int32_t t = threadIdx.x; t < nslots; t += blockDim.x)
                ridx[t] = qinv_of(P, mod_M(r0 - (W - 1) + t - j0m, kshM, P.fd_M));
            __syncthreads();
        }

        // ---- load: cp.async of every staged row's 16-byte hull --------------------------
        // Source row of slot t: contiguous (rowbase + t) mod M for ROT / C2R / COPY,
        // ridx[t] for R2C.
        const int32_t rowbase = MODE == COL_ROT ? mod_M(r0 + base_off, kshM, P.fd_M) : r0;
        const char *Aj = A + static_cast<int64_t>(j0) * EB;
        const uint32_t sst = smem_u32(stage);
        const int32_t nch = nslots * CH;
        for (int32_t e = threadIdx.x; e < nch; e += blockDim.x) {
            const int32_t t = e / CH, k = e - t * CH;
            int32_t row;
            if (MODE == COL_R2C_SHUF) {
                row = ridx[t];
            } else {
                row = rowbase + t;
                if (row >= P.M) row = row - P.M < P.M ? row - P.M : mod_M(row, kshM, P.fd_M);
            }
            const char *ra = Aj + row * pitch;
            const int d = static_cast<int>(reinterpret_cast<uintptr_t>(ra) & 15);
            if (k == 0) dlt[t] = static_cast<uint8_t>(d);
            const char *lo = ra - d + 16 * k;
            if (16 * k >= d + Wt * EB) continue;  // past the end of this row's tile
            const uint32_t dst = sst + t * SLOT + 16 * k;
            // Only row 0's head and row M-1's tail can leave the matrix.
            if ((row != 0 && row != P.M - 1) || (lo >= A && lo + 16 <= Aend)) {
                cp_async16(dst, lo);
            } else {
#pragma unroll
                for (int q = 0; q < 16; q += EB)
                    if (lo + q >= A && lo + q < Aend) cp_async_small<EB>(dst + q, lo + q);
            }
        }

        // ---- C2R: destination rows of the band, while the loads are in flight --------
        if (MODE == COL_C2R_SHUF) {
            for (int32_t kk = threadIdx.x; kk < nrows; kk += blockDim.x)
                ridx[kk] = qinv_of(P, mod_M(r0 + kk - j0m, kshM, P.fd_M));
        }
        cp_async_wait_all();

        // In-place hazard barrier: the whole tile has been read before anyone writes it.
        if (use_barrier) group_barrier(ctr, (++nbar) * static_cast<unsigned int>(P.G));
        else __syncthreads();

        // ---- write -----------------------------------------------------------------------
        const int32_t w = threadIdx.x & (W - 1);  // blockDim is a multiple of W: fixed per thread
        if (w < Wt) {
            int32_t dw = 0;
            if (MODE == COL_ROT) {
                const int32_t qw = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + w), P.fd_b));
                dw = P.rot_sign > 0 ? qw - lo_q : hi_q - qw;  // rho_w - min rho
            } else if (MODE == COL_C2R_SHUF) {
                dw = w;
            } else if (MODE == COL_R2C_SHUF) {
                dw = W - 1 - w;
            }
            T *out = reinterpret_cast<T *>(A) + j0 + w;
            const unsigned char *sw = stage + dw * SLOT + w * EB;
            const uint8_t *dl = dlt + dw;
            const int32_t kstep = blockDim.x >> LW;
#pragma unroll 4
            for (int32_t kk = threadIdx.x >> LW; kk < nrows; kk += kstep) {
                const T v = *reinterpret_cast<const T *>(sw + kk * SLOT + dl[kk]);
                const int64_t orow = MODE == COL_C2R_SHUF ? ridx[kk] : r0 + kk;
                out[orow * P.N] = v;
            }
        }
        __syncthreads();  // shared memory is refilled for the next tile
    }
}

template <int EB, int MODE, int TWB>
void *kptr() {
    return reinterpret_cast<void *>(col_tile_kernel<EB, MODE, TWB>);
}

template <int EB, int TWB>
void *col_kernel_w(int mode) {
    switch (mode) {
        case COL_ROT: return kptr<EB, COL_ROT, TWB>();
        case COL_C2R_SHUF: return kptr<EB, COL_C2R_SHUF, TWB>();
        case COL_R2C_SHUF: return kptr<EB, COL_R2C_SHUF, TWB>();
        case COL_COPY: return kptr<EB, COL_COPY, TWB>();
        default: return nullptr;
    }
}

template <int EB>
void *col_kernel_e(int mode, int twb) {
    switch (twb) {
        case 32: return col_kernel_w<EB, 32>(mode);
        case 64: return col_kernel_w<EB, 64>(mode);
        case 128: return col_kernel_w<EB, 128>(mode);
        default: return nullptr;
    }
}

void *col_kernel(int mode, int eb, int twb) {
    switch (eb) {
        case 4: return col_kernel_e<4>(mode, twb);
        case 8: return col_kernel_e<8>(mode, twb);
        case 16: return col_kernel_e<16>(mode, twb);
        default: return nullptr;
    }
}

}  // namespace

size_t col_smem_bytes(int64_t B, int64_t W, int eb) {
    const int64_t twb = W * eb;
    const int64_t nslots = B + W - 1;
    const int64_t slot = twb + 16;
    return static_cast<size_t>(((nslots * (slot + 1) + 3) & ~int64_t(3)) + nslots * 4);
}

int col_block_threads() { return kColThreads; }

int col_resident_ctas(int mode, int eb, int twb, size_t smem) {
    void *kern = col_kernel(mode, eb, twb);
    if (!kern || ensure_kernel_attrs(kern, smem, false) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return cached_resident_blocks(kern, kColThreads, smem);
}

cudaError_t launch_col(const ColParams &P0, int mode, int eb, cudaStream_t st, size_t smem) {
    void *kern = col_kernel(mode, eb, P0.W * eb);
    if (!kern) return cudaErrorInvalidValue;
    cudaError_t e = ensure_kernel_attrs(kern, smem, false);
    if (e != cudaSuccess) return e;
    ColParams P = P0;
    const bool need_ctr = P.G > 1;
    if (need_ctr) {
        // One arrival counter per group, stream-ordered scratch (freed after the launch).
        e = cudaMallocAsync(reinterpret_cast<void **>(&P.ctr), sizeof(unsigned int) * P.ngroups, st);
        if (e != cudaSuccess) return e;
        e = cudaMemsetAsync(P.ctr, 0, sizeof(unsigned int) * P.ngroups, st);
        if (e != cudaSuccess) return e;
    }
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    cfg.gridDim = dim3(static_cast<unsigned>(P.ngroups) * static_cast<unsigned>(P.G));
    cfg.blockDim = dim3(kColThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    attr[0].id = cudaLaunchAttributeCooperative;  // all CTAs co-resident: the group spin is safe
    attr[0].val.cooperative = need_ctr ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    void *args[] = {&P};
    e = cudaLaunchKernelExC(&cfg, kern, args);
    if (need_ctr) {
        cudaError_t e2 = cudaFreeAsync(P.ctr, st);
        if (e == cudaSuccess) e = e2;
    }
    return e;
}

}  // namespace ipt
