// Column-tile kernel (§3 Eqs. 23, 26, §4.1-4.3,
// §4.6-4.7).
//
// A column operation permutes every column independently.  The B200 realisation stages a
// whole column tile -- all M rows x W adjacent columns (TWB = W * eb = 128 bytes wide) --
// on chip, spread over the shared memory of a GROUP of G CTAs (member r owns the output
// band [r B, r B + B)), and makes the operation a single read + write pass.  In-place
// safety: every member finishes reading its part of the tile before ANY member writes (a
// per-tile barrier in global memory: release-add on a counter, acquire spin until all G
// members arrived); tiles are disjoint byte ranges owned by exactly one group.  This
// replaces the paper's multi-pass cache-aware rotate (coarse cycle following + fine
// on-chip rotation, §4.6) and cycle-following row permute (§4.7) -- prior art for a K20c.
//
// Tile-local forms (w = j - j0 is the column inside the tile [j0, j0 + W); "slot" t is the
// t-th input row a member reads; output row k of the band is written to global row o(k)):
//  * COL_ROT, gather rotation rho_j = sign * floor(j/b) (Eq. 23, sign = +1: the C2R
//    pre-rotation; Eq. 36, sign = -1: the R2C post-rotation):
//        out[i][w] = in[(i + rho_{j0+w}) mod M][w]
//    slots = input rows r0 + min rho + t (contiguous, cyclic); slot t, column w feeds
//    band row k = t - (rho_w - min rho); o(k) = r0 + k.  rho varies by < W in a tile
//    (the residual bound of :767-773).
//  * COL_C2R_SHUF, s'_j(i) = (j + q(i)) mod M (Eq. 26 = p_j o q, Eqs. 32-33):
//        out[i][w] = in[(k + w) mod M][w],  k = (j0 + q(i)) mod M,
//    scatter form: slots = rows r0 + t (band + W-1 halo rows), slot t column w feeds the
//    skewed row k = t - w, which is output row o(k) = q^{-1}((r0 + k - j0) mod M) (Eq. 34).
//  * COL_R2C_SHUF, (s')^{-1}_j(i) = q^{-1}((i - j) mod M) (Eqs. 34-35):
//        out[i][w] = in[q^{-1}((i - w - j0) mod M)][w],
//    slots = rows q^{-1}((r0 - W + 1 + t - j0) mod M) (scattered), slot t column w feeds
//    k = t - (W - 1) + w; o(k) = r0 + k.
//  * COL_COPY: identity (measurement hook).
//
// Data path (lane = tile column, see col_tile_kernel): element-granular cp.async from each
// 128-byte tile row straight into the element's OUTPUT row in shared memory -- the skew /
// rotation / permutation is the copy's destination address -- then whole output rows
// written back with coalesced element stores.  Earlier variants, all slower and kept in
// the round-1 notes (profiles/): 16-byte cp.async hulls + per-element skewed gathers
// (54 instr/element), 128-bit register loads + shared-memory scatter, TMA bulk copies.
//
// Why software groups rather than hardware clusters: a group can be any size up to the
// co-resident CTA count (a 17226-row tile of 128 B is ~2.2 MB, beyond a 16-CTA cluster),
// and the non-persistent grid lets CTAs drift out of lock-step (a persistent cooperative
// variant and a two-buffer pipelined variant were both slower: profiles/).  The grid is one
// CTA per (tile, band); see col_tile_kernel for why the spin barrier cannot deadlock.
#include "plan.h"

namespace ipt {

namespace {

#ifndef IPT_COL_THREADS
#define IPT_COL_THREADS 512
#endif
constexpr int kColThreads = IPT_COL_THREADS;

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

// Group barrier in global memory: counter ctr counts arrivals of all tiles sharing it.
__device__ __forceinline__ void group_barrier(unsigned int *ctr, unsigned int target) {
    __syncthreads();  // every thread's staged data is in shared memory
    if (threadIdx.x == 0) {
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
        unsigned int v;
        while (true) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
            if (v >= target) break;
            __nanosleep(128);
        }
    }
    __syncthreads();
}

// Shared-memory layout: [orow B*4 | srow nslots*4 | rows B*TWB].
__host__ __device__ inline size_t al16(size_t x) { return (x + 15) & ~size_t(15); }
__host__ __device__ inline size_t smem_layout(int64_t B, int W, int twb, size_t *off_srow, size_t *off_rows) {
    const size_t nslots = static_cast<size_t>(B) + W - 1;
    size_t o = al16(static_cast<size_t>(B) * 4);
    *off_srow = o;
    o += al16(nslots * 4);
    *off_rows = o;
    return o + static_cast<size_t>(B) * twb;
}

template <int EB>
__device__ __forceinline__ void cp_async_elem(uint32_t dst, const void *src) {
    if constexpr (EB == 16)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(src) : "memory");
    else
        asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" :: "r"(dst), "l"(src), "n"(EB) : "memory");
}

// One CTA per (tile, band).  The CTA's logical id comes from a ticket counter taken at
// start (dispatch order), so the G members of a tile are exactly G consecutive tickets:
// every group whose tickets are all taken is fully resident, hence only the newest group
// can be waiting for members, and those get scheduled as older groups finish -- the spin
// barrier cannot deadlock as long as one group fits on the GPU (G <= resident CTAs).
//
// Thread mapping: lane = tile column w (W = TWB/eb lanes per tile row, 32/W rows per warp
// instruction).  A load instruction copies whole tile rows (128 contiguous bytes) with
// element-granular cp.async, each element landing directly in its OUTPUT row of the band in
// shared memory (row k = t - dw[w]): the skew / rotation is done by the copy's
// destination address, and the bank of every element is its column (conflict-free).  A
// store instruction writes whole output rows (128 contiguous bytes).  No 16-byte alignment
// is needed anywhere: element accesses work at every row phase and never leave the tile.
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void col_tile_one(const ColParams &P, unsigned char *smem, uint32_t tt, int32_t r) {
    using T = typename Word<EB>::T;
    constexpr int W = TWB / EB;
    constexpr int RPW = 32 / W;  // tile rows per warp instruction
    const int32_t r0 = r * P.B;
    const int32_t nrows = max(0, min(P.M, r0 + P.B) - r0);
    const bool use_barrier = P.G > 1 && !(MODE == COL_COPY && P.rot_sign == 0);
    const uint32_t kshM = P.kshM;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;

    // ---- tile geometry --------------------------------------------------------------
    const uint32_t mat = fdiv(tt, P.fd_nt);
    const int32_t tile = static_cast<int32_t>(tt - mat * static_cast<uint32_t>(P.ntiles));
    char *A = P.base + static_cast<int64_t>(mat) * P.mat_stride_bytes;
    const int32_t j0 = tile * W;
    const int32_t Wt = min(W, P.N - j0);
    const int32_t j0m = static_cast<int32_t>(fmod_(static_cast<uint32_t>(j0), P.fd_M));
    int32_t ext = W - 1, lo_q = 0, hi_q = 0, base_off = 0;
    if (MODE == COL_ROT) {
        lo_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0), P.fd_b));
        hi_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + Wt - 1), P.fd_b));
        ext = hi_q - lo_q;
        base_off = P.rot_sign > 0 ? lo_q : -hi_q;  // smallest rotation amount in the tile
        // Columns j < b rotate by 0 (Eq. 23): a tile made only of them is left alone.  The
        // skip is group-uniform; still arrive, later tiles sharing the counter count it.
        if (hi_q == 0) {
            if (use_barrier && threadIdx.x == 0) atomicAdd(P.ctr + (tt % kCtrSlots), 1u);
            return;
        }
    } else if (MODE == COL_COPY) {
        ext = 0;
    }
    const int32_t nslots = nrows > 0 ? nrows + ext : 0;

    size_t o_srow, o_rows;
    smem_layout(P.B, W, TWB, &o_srow, &o_rows);
    int32_t *orow = reinterpret_cast<int32_t *>(smem);
    int32_t *srow = reinterpret_cast<int32_t *>(smem + o_srow);
    unsigned char *rows = smem + o_rows;
    char *Aj = A + static_cast<int64_t>(j0) * EB;

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    const int w = lane % W, sub = lane / W;
    int32_t dw = 0;  // slot t, column w feeds band row k = t - dw
    if (MODE == COL_ROT) {
        const int32_t qw = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + min(w, Wt - 1)), P.fd_b));
        dw = P.rot_sign > 0 ? qw - lo_q : hi_q - qw;  // rho_w - min rho
    } else if (MODE == COL_C2R_SHUF) {
        dw = w;
    } else if (MODE == COL_R2C_SHUF) {
        dw = W - 1 - w;
    }

    // ---- pre-pass: scattered row indices (C2R destinations, R2C sources) --------------
    if (MODE == COL_C2R_SHUF) {
        for (int32_t k = threadIdx.x; k < nrows; k += blockDim.x)
            orow[k] = qinv_of(P, mod_M(r0 + k - j0m, kshM, P.fd_M));
    }
    if (MODE == COL_R2C_SHUF) {
        for (int32_t t = threadIdx.x; t < nslots; t += blockDim.x)
            srow[t] = qinv_of(P, mod_M(r0 - (W - 1) + t - j0m, kshM, P.fd_M));
        __syncthreads();
    }

    // ---- load: every element straight to its output row -------------------------------
    const int32_t rowbase = MODE == COL_ROT ? mod_M(r0 + base_off, kshM, P.fd_M) : r0;
    const uint32_t srows = static_cast<uint32_t>(__cvta_generic_to_shared(rows)) + w * EB;
    char *colp = Aj + w * EB;
    char *tmpw = P.tmp + static_cast<int64_t>(j0 + w) * EB;  // skinny engine only
    const int32_t step = nwarps * RPW;  // slots between a lane's consecutive rows
    const int32_t t0 = warp * RPW + sub;
    if (w < Wt && P.remap < 0) {  // skinny: row s is stored at s-1, row 0 in tmp
        int32_t t = t0;
        if (t < dw) t += ((dw - t + step - 1) / step) * step;
        for (; t < dw + nrows; t += step) {
            const int32_t s = MODE == COL_R2C_SHUF ? srow[t] : mod_M(rowbase + t, kshM, P.fd_M);
            cp_async_elem<EB>(srows + (t - dw) * TWB, s == 0 ? tmpw : colp + (s - 1) * pitch);
        }
    } else if (w < Wt) {
        // This lane's slots t with 0 <= k = t - dw < nrows (the others are halo elements no
        // band row needs): a branch-free walk with incremental shared and global addresses.
        int32_t t = t0;
        if (t < dw) t += ((dw - t + step - 1) / step) * step;
        const int32_t tend = dw + nrows;
        uint32_t sa = srows + (t - dw) * TWB;
        const uint32_t sa_inc = step * TWB;
        if (MODE == COL_R2C_SHUF) {
#pragma unroll 4
            for (; t < tend; t += step, sa += sa_inc) cp_async_elem<EB>(sa, colp + srow[t] * pitch);
        } else if (step <= P.M) {
            int32_t s = mod_M(rowbase + t, kshM, P.fd_M);
            const char *g = colp + s * pitch;
            const int64_t g_inc = step * pitch, g_wrap = static_cast<int64_t>(P.M) * pitch;
#pragma unroll 4
            for (; t < tend; t += step, sa += sa_inc) {
                cp_async_elem<EB>(sa, g);
                s += step;
                g += g_inc;
                if (s >= P.M) {
                    s -= P.M;
                    g -= g_wrap;
                }
            }
        } else {  // tiny M: fewer rows than one step
            for (; t < tend; t += step, sa += sa_inc)
                cp_async_elem<EB>(sa, colp + mod_M(rowbase + t, kshM, P.fd_M) * pitch);
        }
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");

    // In-place hazard barrier: the whole tile has been read before anyone writes it.
    // Counter slot tt mod kCtrSlots, monotone over the tiles that share it.
    if (use_barrier) {
        const unsigned int slot = tt % kCtrSlots;  // power of two
        const unsigned int target = (tt / kCtrSlots + 1) * static_cast<unsigned int>(P.G);
        group_barrier(P.ctr + slot, target);
    } else {
        __syncthreads();
    }

    // ---- store: whole output rows -------------------------------------------------------
    if (w < Wt) {
        const unsigned char *sr = rows + w * EB;
        int32_t k = t0;
        if (P.remap > 0) {  // skinny: output row o is stored at o+1, row M-1 in tmp
            for (; k < nrows; k += step) {
                const int32_t o = MODE == COL_C2R_SHUF ? orow[k] : r0 + k;
                *reinterpret_cast<T *>(o == P.M - 1 ? tmpw : colp + static_cast<int64_t>(o + 1) * pitch) =
                    *reinterpret_cast<const T *>(sr + k * TWB);
            }
        } else if (MODE == COL_C2R_SHUF) {
#pragma unroll 4
            for (; k < nrows; k += step)
                *reinterpret_cast<T *>(colp + static_cast<int64_t>(orow[k]) * pitch) =
                    *reinterpret_cast<const T *>(sr + k * TWB);
        } else {
            char *g = colp + static_cast<int64_t>(r0 + k) * pitch;
            const int64_t g_inc = step * pitch;
#pragma unroll 4
            for (; k < nrows; k += step, g += g_inc) *reinterpret_cast<T *>(g) = *reinterpret_cast<const T *>(sr + k * TWB);
        }
    }
}

template <int EB, int MODE, int TWB>
__global__ void __launch_bounds__(kColThreads) col_tile_kernel(ColParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ unsigned int s_ticket;
    if (threadIdx.x == 0) s_ticket = atomicAdd(P.ctr + kTicketSlot, 1u);
    __syncthreads();
    const unsigned int ticket = s_ticket;
    if (P.G == 1) {  // a tile fits one CTA: no barrier, P.tpc consecutive tiles per CTA
        const uint64_t t_end = min(static_cast<uint64_t>(P.total_tiles), (static_cast<uint64_t>(ticket) + 1) * P.tpc);
        for (uint64_t tt = static_cast<uint64_t>(ticket) * P.tpc; tt < t_end; ++tt) {
            col_tile_one<EB, MODE, TWB>(P, smem, static_cast<uint32_t>(tt), 0);
            __syncthreads();  // shared memory is reused by the next tile
        }
        return;
    }
    const uint32_t tt = fdiv(ticket, P.fd_G);                  // tile (of all matrices)
    const int32_t r = static_cast<int32_t>(ticket - tt * P.G);  // band
    col_tile_one<EB, MODE, TWB>(P, smem, tt, r);
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
    size_t a, b;
    return smem_layout(B, static_cast<int>(W), static_cast<int>(W * eb), &a, &b);
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
    const int64_t grid = P.G == 1 ? (P.total_tiles + P.tpc - 1) / P.tpc : P.total_tiles * P.G;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    // Ticket + group counters: the stream's own block, zeroed in stream order.
    P.ctr = group_counters(st, kCtrSlots + 1);
    if (!P.ctr) return cudaErrorMemoryAllocation;
    e = cudaMemsetAsync(P.ctr, 0, sizeof(unsigned int) * (kTicketSlot + 1), st);
    if (e != cudaSuccess) return e;
    void *args[] = {&P};
    return cudaLaunchKernel(kern, dim3(static_cast<unsigned>(grid)), dim3(kColThreads), args, smem, st);
}

}  // namespace ipt
