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
// Why software groups rather than hardware clusters: a group can be any size up to the
// co-resident CTA count (a 17226-row tile of 128 B is ~2.6 MB, beyond a 16-CTA cluster
// at 128-byte tiles), and the non-persistent grid lets CTAs drift out of lock-step (a
// persistent cooperative variant and a two-buffer pipelined variant were both slower:
// profiles/).  The grid is one CTA per (tile, band); see col_tile_kernel for why the spin
// barrier cannot deadlock.
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
// element by element.  (One TMA bulk copy per 144-byte hull was tried and is ~2x slower:
// the TMA engine does not keep up with that many tiny requests; profiles/.)  Stores: one 16-byte destination
// chunk per thread, gathered from the staged rows and written with a vector store
// (element stores only in a row's ragged head/tail chunk).
#include "plan.h"

namespace ipt {

namespace {

#ifndef IPT_COL_THREADS
#define IPT_COL_THREADS 512
#endif
constexpr int kColThreads = IPT_COL_THREADS;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
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

// Per-tile geometry of one staging buffer.
struct TileCtx {
    char *A;            // this matrix
    const char *Aend;
    int32_t j0, Wt, j0m;
    int32_t lo_q, hi_q, base_off, nslots;
};

// Staging buffer layout (one of two): [dw W*4 | stage nslots_max*SLOT | dlt nslots_max |
// ridx nslots_max*4], nslots_max = B + W - 1.
template <int TWB>
__host__ __device__ constexpr size_t buf_dw_bytes(int W) { return (static_cast<size_t>(W) * 4 + 15) & ~size_t(15); }
__host__ __device__ inline size_t buf_bytes(int64_t nslots_max, int W, int twb) {
    const size_t slot = static_cast<size_t>(twb) + 16;
    return ((static_cast<size_t>(W) * 4 + 15) & ~size_t(15)) + ((static_cast<size_t>(nslots_max) * (slot + 1) + 15) & ~size_t(15)) +
           ((static_cast<size_t>(nslots_max) * 4 + 15) & ~size_t(15));  // keeps the second buffer 16-B aligned
}

template <int EB, int MODE, int TWB>
__device__ __forceinline__ bool make_ctx(const ColParams &P, int64_t tt, int32_t nrows, TileCtx &c) {
    constexpr int W = TWB / EB;
    const int32_t tile = static_cast<int32_t>(tt % P.ntiles);
    const int64_t mat = tt / P.ntiles;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    c.A = P.base + mat * P.mat_stride_bytes;
    c.Aend = c.A + static_cast<int64_t>(P.M) * pitch;
    c.j0 = tile * W;
    c.Wt = min(W, P.N - c.j0);
    c.j0m = static_cast<int32_t>(fmod_(static_cast<uint32_t>(c.j0), P.fd_M));
    int32_t ext = W - 1;
    c.lo_q = c.hi_q = c.base_off = 0;
    if (MODE == COL_ROT) {
        c.lo_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(c.j0), P.fd_b));
        c.hi_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(c.j0 + c.Wt - 1), P.fd_b));
        // Columns j < b rotate by 0 (Eq. 23): a tile made only of them is left alone.
        // Every member sees the same tile, so the skip is group-uniform.
        if (c.hi_q == 0) return false;
        ext = c.hi_q - c.lo_q;
        c.base_off = P.rot_sign > 0 ? c.lo_q : -c.hi_q;  // smallest rotation amount in the tile
    } else if (MODE == COL_COPY) {
        ext = 0;
    }
    c.nslots = nrows > 0 ? nrows + ext : 0;
    return true;
}

template <int EB, int MODE, int TWB>
__device__ __forceinline__ int64_t next_tile(const ColParams &P, int64_t tt, int32_t nrows, TileCtx &c) {
    for (; tt < P.total_tiles; tt += P.ngroups)
        if (make_ctx<EB, MODE, TWB>(P, tt, nrows, c)) return tt;
    return tt;
}

// Issue the cp.async loads of one tile band into buffer `buf` (one commit group).
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void load_tile(const ColParams &P, const TileCtx &c, unsigned char *buf, int32_t r0,
                                          int32_t nrows, int32_t nslots_max, uint32_t kshM) {
    constexpr int W = TWB / EB;
    constexpr int SLOT = TileGeom<TWB>::SLOT;
    constexpr int CH = TileGeom<TWB>::CH;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    int32_t *dwt = reinterpret_cast<int32_t *>(buf);
    unsigned char *stage = buf + buf_dw_bytes<TWB>(W);
    uint8_t *dlt = stage + static_cast<size_t>(nslots_max) * SLOT;
    int32_t *ridx = reinterpret_cast<int32_t *>(stage + ((static_cast<size_t>(nslots_max) * (SLOT + 1) + 15) & ~size_t(15)));

    // Slot offset of column w: the element of output row kk comes from staged row kk + dw[w].
    for (int32_t w = threadIdx.x; w < W; w += blockDim.x) {
        int32_t dw = 0;
        if (MODE == COL_ROT) {
            const int32_t qw = static_cast<int32_t>(fdiv(static_cast<uint32_t>(c.j0 + min(w, c.Wt - 1)), P.fd_b));
            dw = P.rot_sign > 0 ? qw - c.lo_q : c.hi_q - qw;  // rho_w - min rho
        } else if (MODE == COL_C2R_SHUF) {
            dw = w;
        } else if (MODE == COL_R2C_SHUF) {
            dw = W - 1 - w;
        }
        dwt[w] = dw;
    }
    // Source row of slot t: contiguous (rowbase + t) mod M for ROT / C2R / COPY,
    // q^{-1}((r0 - W + 1 + t - j0) mod M) for R2C (ridx, computed first).
    if (MODE == COL_R2C_SHUF) {
        for (int32_t t = threadIdx.x; t < c.nslots; t += blockDim.x)
            ridx[t] = qinv_of(P, mod_M(r0 - (W - 1) + t - c.j0m, kshM, P.fd_M));
        __syncthreads();
    }
    const int32_t rowbase = MODE == COL_ROT ? mod_M(r0 + c.base_off, kshM, P.fd_M) : r0;
    const char *Aj = c.A + static_cast<int64_t>(c.j0) * EB;
    const uint32_t sst = smem_u32(stage);
    const int32_t nch = c.nslots * CH;
    const int32_t vbytes = c.Wt * EB;
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
        if (16 * k >= d + vbytes) continue;  // past the end of this row's tile
        const char *lo = ra - d + 16 * k;
        const uint32_t dst = sst + t * SLOT + 16 * k;
        // Only row 0's head and row M-1's tail can leave the matrix.
        if ((row != 0 && row != P.M - 1) || (lo >= c.A && lo + 16 <= c.Aend)) {
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(lo) : "memory");
        } else {
#pragma unroll
            for (int q = 0; q < 16; q += EB)
                if (lo + q >= c.A && lo + q < c.Aend) cp_async_small<EB>(dst + q, lo + q);
        }
    }
    // C2R: destination rows of the band, while the loads are in flight.
    if (MODE == COL_C2R_SHUF) {
        for (int32_t kk = threadIdx.x; kk < nrows; kk += blockDim.x)
            ridx[kk] = qinv_of(P, mod_M(r0 + kk - c.j0m, kshM, P.fd_M));
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// Write one tile band from buffer `buf`: one 16-byte destination chunk per thread.
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void store_tile(const ColParams &P, const TileCtx &c, const unsigned char *buf, int32_t r0,
                                           int32_t nrows, int32_t nslots_max) {
    using T = typename Word<EB>::T;
    constexpr int W = TWB / EB;
    constexpr int SLOT = TileGeom<TWB>::SLOT;
    constexpr int NQ = TWB / 16 + 1;  // 16-byte destination chunks a tile row can touch
    constexpr int PER = 16 / EB;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    const int32_t *dwt = reinterpret_cast<const int32_t *>(buf);
    const unsigned char *stage = buf + buf_dw_bytes<TWB>(W);
    const uint8_t *dlt = stage + static_cast<size_t>(nslots_max) * SLOT;
    const int32_t *ridx =
        reinterpret_cast<const int32_t *>(stage + ((static_cast<size_t>(nslots_max) * (SLOT + 1) + 15) & ~size_t(15)));
    char *Aj = c.A + static_cast<int64_t>(c.j0) * EB;
    const int32_t Wt = c.Wt;
    const int32_t nout = nrows * NQ;
    for (int32_t e = threadIdx.x; e < nout; e += blockDim.x) {
        const int32_t kk = e / NQ, q = e - kk * NQ;
        const int64_t orow = MODE == COL_C2R_SHUF ? ridx[kk] : r0 + kk;
        char *da = Aj + orow * pitch;  // output row's tile start
        const int dd = static_cast<int>(reinterpret_cast<uintptr_t>(da) & 15);
        const int w0 = (16 * q - dd) / EB;  // first column of this chunk (may be < 0)
        if (w0 >= Wt) continue;
        if (w0 >= 0 && w0 + PER <= Wt) {
            union { uint4 u; T t[PER]; } v;
            const int32_t ta = kk + dwt[w0], tb = kk + dwt[w0 + PER - 1];
            const uint32_t so = ta * SLOT + dlt[ta] + w0 * EB;
            if (ta == tb && (so & 15) == 0) {  // one staged row, aligned: a single LDS.128
                v.u = *reinterpret_cast<const uint4 *>(stage + so);
            } else {
#pragma unroll
                for (int x = 0; x < PER; ++x) {
                    const int32_t t = kk + dwt[w0 + x];
                    v.t[x] = *reinterpret_cast<const T *>(stage + t * SLOT + dlt[t] + (w0 + x) * EB);
                }
            }
            *reinterpret_cast<uint4 *>(da + w0 * EB) = v.u;
        } else {
#pragma unroll
            for (int x = 0; x < PER; ++x) {
                const int w = w0 + x;
                if (w < 0 || w >= Wt) continue;
                const int32_t t = kk + dwt[w];
                reinterpret_cast<T *>(da)[w] = *reinterpret_cast<const T *>(stage + t * SLOT + dlt[t] + w * EB);
            }
        }
    }
}

// One CTA per (tile, band).  The CTA's logical id comes from a ticket counter taken at
// start (dispatch order), so the G members of a tile are exactly G consecutive tickets:
// every group whose tickets are all taken is fully resident, hence only the newest group
// can be waiting for members, and those get scheduled as older groups finish -- the spin
// barrier cannot deadlock as long as one group fits on the GPU (G <= resident CTAs).
template <int EB, int MODE, int TWB>
__global__ void __launch_bounds__(kColThreads) col_tile_kernel(ColParams P) {
    constexpr int W = TWB / EB;
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ unsigned int s_ticket;
    if (threadIdx.x == 0) s_ticket = atomicAdd(P.ctr + kTicketSlot, 1u);
    __syncthreads();
    const unsigned int ticket = s_ticket;
    const int64_t tt = ticket / static_cast<unsigned int>(P.G);   // tile (of all matrices)
    const int32_t r = static_cast<int32_t>(ticket - tt * P.G);     // band
    const int32_t r0 = r * P.B;
    const int32_t r1 = min(P.M, r0 + P.B);
    const int32_t nrows = max(0, r1 - r0);
    const int32_t nslots_max = P.B + W - 1;
    const uint32_t kshM = static_cast<uint32_t>(2 + W / P.M) * static_cast<uint32_t>(P.M);
    const bool use_barrier = P.G > 1 && !(MODE == COL_COPY && P.rot_sign == 0);

    TileCtx c;
    if (!make_ctx<EB, MODE, TWB>(P, tt, nrows, c)) {  // group-uniform skip (ROT amount 0)
        // Still arrive: later tiles sharing this counter slot count these arrivals.
        if (use_barrier && threadIdx.x == 0)
            atomicAdd(P.ctr + static_cast<unsigned int>(tt % kCtrSlots), 1u);
        return;
    }
    load_tile<EB, MODE, TWB>(P, c, smem, r0, nrows, nslots_max, kshM);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    // In-place hazard barrier: the whole tile has been read before anyone writes it.
    // Counter slot tt mod kCtrSlots, monotone over the tiles that share it.
    if (use_barrier) {
        const unsigned int slot = static_cast<unsigned int>(tt % kCtrSlots);
        const unsigned int target = static_cast<unsigned int>(tt / kCtrSlots + 1) * static_cast<unsigned int>(P.G);
        group_barrier(P.ctr + slot, target);
    } else {
        __syncthreads();
    }
    store_tile<EB, MODE, TWB>(P, c, smem, r0, nrows, nslots_max);
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
    return buf_bytes(B + W - 1, static_cast<int>(W), static_cast<int>(W * eb));
}

int64_t col_max_band(int64_t W) { return (int64_t(1) << 24) - W; }

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
    const int64_t grid = P.total_tiles * P.G;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    // Ticket + group counters: the stream's own block, zeroed in stream order.
    P.ctr = group_counters(st, kCtrSlots + 1);
    if (!P.ctr) return cudaErrorMemoryAllocation;
    const int64_t used = P.total_tiles < kCtrSlots ? P.total_tiles : kCtrSlots;
    e = cudaMemsetAsync(P.ctr, 0, sizeof(unsigned int) * (kTicketSlot + 1), st);
    if (e != cudaSuccess) return e;
    (void)used;
    void *args[] = {&P};
    return cudaLaunchKernel(kern, dim3(static_cast<unsigned>(grid)), dim3(kColThreads), args, smem, st);
}

}  // namespace ipt
