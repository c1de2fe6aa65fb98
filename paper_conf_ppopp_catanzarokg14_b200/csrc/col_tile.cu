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
#include <algorithm>

#include "plan.h"

namespace ipt {

namespace {

#ifndef IPT_COL_THREADS
#define IPT_COL_THREADS 512
#endif
constexpr int kColThreads = IPT_COL_THREADS;
constexpr int kMaxColBufs = 4;  // unit buffers per CTA of the pipelined kernel

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

// Shared-memory layout of one unit buffer:
//   [orow B*8 | srow nslots*4 | sbase nslots*4 | rows]   (orow: C2R output row byte offsets)
// rows: nslots input rows ("slots") of HS = TWB + 16 bytes, each the 16-byte-aligned hull
// of its tile row; sbase[t] = shared address of slot t's first tile element.
__host__ __device__ inline size_t al16(size_t x) { return (x + 15) & ~size_t(15); }
struct SmemLayout {
    size_t srow, sbase, rows, total;
};
__host__ __device__ constexpr int hull_pitch(int twb) { return twb + 16; }
__host__ __device__ inline SmemLayout smem_layout(int64_t B, int W, int twb, int eb) {
    (void)eb;
    const size_t nslots = static_cast<size_t>(B) + W - 1;
    SmemLayout L;
    size_t o = al16(static_cast<size_t>(B) * 8);
    L.srow = o;
    o += al16(nslots * 4);
    L.sbase = o;
    o += al16(nslots * 4);
    L.rows = o;  // the kernels round the slot region up to 128 bytes (TMA destinations): slack below
    // cp.async hulls: nslots x (TWB + 16); TMA: whole boxes of kTmaBoxRows x TWB (+ 3 slots of
    // gather4 padding)
    const size_t hull = nslots * static_cast<size_t>(hull_pitch(twb));
    // (up to 4 phases of super-rows, each rounded up to whole boxes)
    const size_t tma = (((nslots + 3 + kTmaBoxRows - 1) / kTmaBoxRows) * kTmaBoxRows + 4 * kTmaBoxRows) *
                       static_cast<size_t>(twb);
    L.total = o + (hull > tma ? hull : tma) + 128;
    return L;
}

// One column-tile work unit: band r of tile tt (of all matrices).
struct Unit {
    char *inp, *outp;   // column j0 of row 0 of the tile's input / output location
    int64_t in_pitch, out_pitch;  // bytes between rows there (N eb, or TWB in the side tile)
    int32_t r0, nrows;  // output band [r0, r0 + nrows)
    int32_t j0, j0m;    // first column of the tile, j0 mod M
    int32_t rowbase;    // first input row (ROT / C2R)
    int32_t lo_q, hi_q; // ROT: floor(j/b) of the tile's first / last column
    int32_t nslots;     // input rows read: band + halo
    int32_t wt;         // columns of this tile (W, or fewer at the ragged right edge)
    bool skip;          // ROT tile made only of columns rotating by 0
};

template <int EB, int MODE, int TWB>
__device__ __forceinline__ Unit unit_make(const ColParams &P, uint32_t tt, int32_t r) {
    constexpr int W = TWB / EB;
    Unit U;
    U.r0 = r * P.B;
    U.nrows = max(0, min(P.M, U.r0 + P.B) - U.r0);
    const uint32_t mat = fdiv(tt, P.fd_nt);
    int32_t tile = static_cast<int32_t>(tt - mat * static_cast<uint32_t>(P.ntiles));
    if (P.lag == LAG_C2R) tile = P.ntiles - 1 - tile;  // right to left
    const int32_t j0 = tile * W;
    U.j0 = j0;
    U.wt = min(W, P.N - j0);
    U.j0m = static_cast<int32_t>(fmod_(static_cast<uint32_t>(j0), P.fd_M));
    U.skip = false;
    U.lo_q = U.hi_q = 0;
    int32_t ext = W - 1, base_off = 0;
    if (MODE == COL_ROT) {
        U.lo_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0), P.fd_b));
        U.hi_q = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j0 + U.wt - 1), P.fd_b));
        ext = U.hi_q - U.lo_q;
        base_off = P.rot_sign > 0 ? U.lo_q : -U.hi_q;  // smallest rotation amount in the tile
        // Columns j < b rotate by 0 (Eq. 23): a tile made only of them is left alone.
        U.skip = U.hi_q == 0;
    } else if (MODE == COL_COPY) {
        ext = 0;
    }
    U.nslots = U.nrows > 0 ? U.nrows + ext : 0;
    U.rowbase = MODE == COL_ROT ? mod_M(U.r0 + base_off, P.kshM, P.fd_M) : U.r0;
    char *A = P.base + static_cast<int64_t>(mat) * P.mat_stride_bytes;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    U.inp = U.outp = A + static_cast<int64_t>(j0) * EB;
    U.in_pitch = U.out_pitch = pitch;
    if (P.lag != LAG_NONE) {
        // Lagged layouts (see "In-place hazard"): tile t >= D lives D tiles to the left,
        // tiles t < D in the side block (columns [t W, t W + W) of its rows).
        const int32_t D = P.lagD;
        char *shifted = tile < D ? side_matrix(P.side, P.sstride, mat, A) + static_cast<int64_t>(tile) * TWB
                                 : A + static_cast<int64_t>(j0 - D * W) * EB;
        const int64_t shifted_pitch = tile < D ? P.spitch : pitch;
        if (P.lag == LAG_R2C) {
            U.outp = shifted;
            U.out_pitch = shifted_pitch;
        } else {
            U.inp = shifted;
            U.in_pitch = shifted_pitch;
        }
    }
    return U;
}

// Slot offset of tile column w: output band row k, column w is slot k + dw(w).
template <int EB, int MODE, int TWB>
__device__ __forceinline__ int32_t dw_of(const ColParams &P, const Unit &U, int32_t w) {
    constexpr int W = TWB / EB;
    if (MODE == COL_C2R_SHUF) return w;
    if (MODE == COL_R2C_SHUF) return W - 1 - w;
    if (MODE == COL_COPY) return 0;
    const int32_t qw = static_cast<int32_t>(fdiv(static_cast<uint32_t>(U.j0 + w), P.fd_b));
    return P.rot_sign > 0 ? qw - U.lo_q : U.hi_q - qw;  // rho_w - min rho
}

// Scattered row indices of a unit, computed by the whole CTA into shared memory:
// C2R destinations orow[k] = q^{-1}((r0 + k - j0) mod M) (Eq. 34; stored as the row's byte
// offset in the output location, so the store loop adds it to the column pointer), R2C sources
// srow[t] = q^{-1}((r0 - W + 1 + t - j0) mod M).  R2C needs a __syncthreads before the load.
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void unit_prepass(const ColParams &P, const Unit &U, int64_t *orow, int32_t *srow,
                                             int nthr) {
    constexpr int W = TWB / EB;
    if (MODE == COL_C2R_SHUF) {
        for (int32_t k = threadIdx.x; k < U.nrows; k += nthr)
            orow[k] = static_cast<int64_t>(qinv_of(P, mod_M(U.r0 + k - U.j0m, P.kshM, P.fd_M))) * U.out_pitch;
    }
    if (MODE == COL_R2C_SHUF) {
        for (int32_t t = threadIdx.x; t < U.nslots; t += nthr)
            srow[t] = qinv_of(P, mod_M(U.r0 - (W - 1) + t - U.j0m, P.kshM, P.fd_M));
    }
}

// Chunks of 16 bytes per tile row: the 16-byte-aligned hull of a TWB-byte row segment
// (one more chunk when the segment is misaligned; 16-byte elements never are).
template <int EB, int TWB> constexpr int chunks_per_row() { return TWB / 16 + (EB < 16 ? 1 : 0); }

template <int EB, int MODE, int TWB, bool EXACT>
__device__ __forceinline__ void unit_load_t(const ColParams &P, const Unit &U, const int32_t *srow, uint32_t *sbase,
                                            uint32_t rows_s, int nthr) {
    constexpr int CPR = chunks_per_row<EB, TWB>();
    constexpr int LPS = CPR < 32 ? CPR : 32;  // lanes per slot
    constexpr int RPI = 32 / LPS;             // slots per warp iteration
    constexpr int CPL = (CPR + 31) / 32;      // chunks per lane
    constexpr int HS = hull_pitch(TWB);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = nthr >> 5;
    const int c = lane % LPS, sub = lane / LPS;
    if (sub >= RPI) return;  // lanes beyond the last whole slot of the warp
    const int32_t step = nwarps * RPI;
    int32_t t = warp * RPI + sub;
    if (t >= U.nslots) return;
    const int64_t pitch = U.in_pitch;
    const int32_t c16 = c * 16;
    uint32_t dst = rows_s + t * HS + c16;
    const uint32_t dst_inc = step * HS;
    uint32_t *sb = sbase + t;
    // Chunks c (+ 32, ...) of slot t's hull; q = the slot's first tile element + 16 c.
    auto issue = [&](const char *q) {
        const uint32_t off = static_cast<uint32_t>(reinterpret_cast<uintptr_t>(q)) & 15u;
        if (c == 0) *sb = dst + off;
#pragma unroll
        for (int k = 0; k < CPL; ++k) {
            if (CPL > 1 && c + 32 * k >= CPR) break;
            const char *src = reinterpret_cast<const char *>(reinterpret_cast<uintptr_t>(q + 512 * k) & ~uintptr_t(15));
            const uint32_t d = dst + 512 * k;
            if (!EXACT) {
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(d), "l"(src) : "memory");
            } else {
                const int32_t rem = U.wt * EB + static_cast<int32_t>(off) - c16 - 512 * k;  // hull bytes from here
                if (rem >= 16) {
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(d), "l"(src) : "memory");
                } else if (rem > 0) {  // row end: read only the tile's bytes (never past the buffer)
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" :: "r"(d), "l"(src), "r"(rem) : "memory");
                }
            }
        }
    };
    if (MODE == COL_R2C_SHUF) {
        for (; t < U.nslots; t += step, dst += dst_inc, sb += step) issue(U.inp + static_cast<int64_t>(srow[t]) * pitch + c16);
    } else if (step <= P.M) {
        // contiguous (cyclic) input rows rowbase + t: incremental row index and pointer
        // Plain pointer walks between the points where a lane's rows wrap past M - 1 (once
        // for big M; small M with a halo longer than M wraps more often).
        int32_t g = mod_M(U.rowbase + t, P.kshM, P.fd_M);
        const char *rp = U.inp + static_cast<int64_t>(g) * pitch + c16;
        const int64_t rp_inc = step * pitch, rp_wrap = static_cast<int64_t>(P.M) * pitch;
        const uint32_t *sb_end = sbase + U.nslots;
        while (sb < sb_end) {
            const int32_t n = (P.M - 1 - g) / step + 1;  // iterations before the wrap
            const uint32_t *stop = sb_end - sb > static_cast<int64_t>(n) * step ? sb + static_cast<int64_t>(n) * step : sb_end;
#pragma unroll 4
            for (; sb < stop; sb += step, dst += dst_inc, rp += rp_inc) issue(rp);
            g += n * step - P.M;
            rp -= rp_wrap;
        }
    } else {  // tiny M: fewer rows than one step
        for (; t < U.nslots; t += step, dst += dst_inc, sb += step)
            issue(U.inp + static_cast<int64_t>(mod_M(U.rowbase + t, P.kshM, P.fd_M)) * pitch + c16);
    }
}

// Load: every input row ("slot" t) is staged as the 16-byte-aligned hull of its tile row
// with 16-byte cp.async (element-granular cp.async runs at ~70% of the 16-byte rate on
// B200 for 4-byte elements: tools/tile_probe.cu); sbase[t] records where its first element
// landed.  The skew / rotation / permutation is applied when the store phase reads shared
// memory.  The rightmost tile of a row (its hull may end past the last byte of the buffer)
// reads exactly the tile's bytes (src-size); every other tile reads whole 16-byte chunks:
// bytes past the tile belong to the next tile of the same row and are never used.  Per slot
// and lane: one 64-bit pointer step, one AND, one cp.async.  Not committed here.
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void unit_load(const ColParams &P, const Unit &U, const int32_t *srow, uint32_t *sbase,
                                          uint32_t rows_s, int nthr) {
    if (U.skip) return;
    if (U.j0 + U.wt >= P.N) unit_load_t<EB, MODE, TWB, true>(P, U, srow, sbase, rows_s, nthr);
    else unit_load_t<EB, MODE, TWB, false>(P, U, srow, sbase, rows_s, nthr);
}

template <int EB>
__device__ __forceinline__ void lds_elem(uint32_t *v, uint32_t a) {
    if constexpr (EB == 4) {
        asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v[0]) : "r"(a));
    } else if constexpr (EB == 8) {
        asm volatile("ld.shared.v2.b32 {%0,%1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(a));
    } else {
        asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(a));
    }
}
template <int EB>
__device__ __forceinline__ void stg_elem(char *p, const uint32_t *v) {
    if constexpr (EB == 4) {
        *reinterpret_cast<uint32_t *>(p) = v[0];
    } else if constexpr (EB == 8) {
        *reinterpret_cast<uint2 *>(p) = make_uint2(v[0], v[1]);
    } else {
        *reinterpret_cast<uint4 *>(p) = make_uint4(v[0], v[1], v[2], v[3]);
    }
}

// Store: lane = tile column w (mod 32: W > 32 columns take W / 32 passes over the row);
// a warp instruction writes min(W, 32) eb contiguous bytes of each of max(1, 32 / W) tile
// rows.  Output band row k goes to global row o(k) (orow[k] for C2R, r0 + k otherwise);
// its element w is slot k + dw(w), read at sbase[slot] + w eb -- for C2R / R2C the lanes
// of a row read a diagonal of the slot array, conflict-free in the banks (slot pitch
// TWB + 16 bytes).
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void unit_store(const ColParams &P, const Unit &U, const int64_t *orow,
                                           const uint32_t *sbase, int nthr) {
    constexpr int W = TWB / EB;
    constexpr int LPR = W < 32 ? W : 32;  // lanes per tile row
    constexpr int RPW = 32 / LPR;         // tile rows per warp instruction
    constexpr int CPL = W / LPR;          // columns per lane
    constexpr int U8 = EB == 16 ? 4 : 8;  // rows in flight per lane (independent shared loads)
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = nthr >> 5;
    const int w0 = lane % LPR, sub = lane / LPR;
    if (U.skip) return;
    const int64_t pitch = U.out_pitch;
    const int32_t step = nwarps * RPW;
#pragma unroll
    for (int cc = 0; cc < CPL; ++cc) {
        const int w = w0 + cc * LPR;
        if (w >= U.wt) break;
        int32_t k = warp * RPW + sub;
        char *colp = U.outp + w * EB;
        const uint32_t *sb = sbase + dw_of<EB, MODE, TWB>(P, U, w);
        const uint32_t wo = w * EB;
        // Batches of U8 rows: all the batch's slot addresses and row offsets first, then its
        // element loads, then its stores -- U8 independent load chains per lane instead of a
        // dependent lds -> lds -> stg chain per row.
        for (; k + (U8 - 1) * step < U.nrows; k += U8 * step) {
            uint32_t a[U8], v[U8][EB / 4];
            int64_t o[U8];
#pragma unroll
            for (int u = 0; u < U8; ++u) {
                a[u] = sb[k + u * step] + wo;
                o[u] = MODE == COL_C2R_SHUF ? orow[k + u * step] : static_cast<int64_t>(U.r0 + k + u * step) * pitch;
            }
#pragma unroll
            for (int u = 0; u < U8; ++u) lds_elem<EB>(v[u], a[u]);
#pragma unroll
            for (int u = 0; u < U8; ++u) stg_elem<EB>(colp + o[u], v[u]);
        }
        for (; k < U.nrows; k += step) {
            uint32_t v[EB / 4];
            lds_elem<EB>(v, sb[k] + wo);
            stg_elem<EB>(colp + (MODE == COL_C2R_SHUF ? orow[k] : static_cast<int64_t>(U.r0 + k) * pitch), v);
        }
    }
}

// Arrival of a unit whose reads have completed (see col_tile_one: relaxed suffices).
__device__ __forceinline__ void group_arrive(unsigned int *ctr) {
    asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
}

// In-place hazard of a column pass, per tile (unit order = ticket order, tile-major):
//  * barrier mode (P.lag == 0): every member of a tile's group reads before any member
//    writes the tile -- each member arrives on the tile's counter once its loads have
//    landed and waits for all G arrivals;
//  * lagged layouts (P.lag != 0; the shuffle passes of two-pass engines): the tile's
//    output location is not its input location.  R2C (LAG_R2C, tiles left to right)
//    writes tile t D tiles to the left (tiles t < D into the side block), where the input
//    of tile t - D lived; C2R (LAG_C2R, tiles right to left) reads tile t from D tiles to
//    the left (tiles t < D from the side block), left there by the lagged row pass, and
//    writes it to its own location, where the input of tile t + D lived.  Either way a
//    unit waits only for the group processed D groups before its own (unit-order tile
//    tt - D; D is chosen so that D groups span about twice the co-resident CTAs, i.e. that
//    group is normally long complete), and the row pass reads / writes the shifted layout
//    (row_shuffle.cu).  Ticket order makes both waits deadlock-free: a waited-for group's
//    members all hold smaller tickets (they are resident or done) and their loads wait on
//    nothing; barrier mode additionally needs G <= co-resident CTAs.
// Counter slot x mod kCtrSlots counts the arrivals of every tile x sharing it (monotone).
__device__ __forceinline__ unsigned int ctr_target(uint32_t x, int G) {
    return (x / kCtrSlots + 1) * static_cast<unsigned int>(G);
}
__device__ __forceinline__ bool ctr_reached(const ColParams &P, uint32_t x) {
    unsigned int v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(P.ctr + (x % kCtrSlots)) : "memory");
    return v >= ctr_target(x, P.G);
}
struct Dep {
    bool arrive;   // arrive on the own tile's counter after the loads
    bool wait;     // wait for the counter of tile `on`
    uint32_t on;
};
template <int MODE>
__device__ __forceinline__ Dep unit_dep(const ColParams &P, uint32_t tt) {
    Dep d;
    if (P.lag) {
        const uint32_t tin = tt - fdiv(tt, P.fd_nt) * static_cast<uint32_t>(P.ntiles);  // position in its matrix
        d.arrive = true;
        d.wait = tin >= static_cast<uint32_t>(P.lagD);
        d.on = tt - P.lagD;
    } else {
        d.arrive = d.wait = P.G > 1 && !(MODE == COL_COPY && P.rot_sign == 0);
        d.on = tt;
    }
    return d;
}

// ---- TMA staging (P.tma; 128-byte tiles, pitch % 16 == 0) -----------------------------
// Slots at a 128-byte pitch (no hull): slot t of the unit at rows_s + 128 t.  C2R / ROT read
// the contiguous rows rowbase .. rowbase + nslots - 1 (units whose rows wrap past M - 1 keep
// cp.async) as 2-D boxes of kTmaBoxRows rows; R2C gathers its scattered rows 4 at a time
// (tile::gather4).  One mbarrier per CTA counts the bytes; out-of-range rows / columns of a
// box (the matrix's last rows, the ragged rightmost tile) are zero-filled by the TMA unit and
// never used.
__device__ __forceinline__ void tmbar_init(uint64_t *bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar)))
                 : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void tmbar_expect(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;"
                 :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tmbar_wait(uint64_t *bar, uint32_t parity) {
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
    asm volatile("{\n .reg .pred p;\n TW_%=:\n"
                 " mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], %1;\n"
                 " @!p bra TW_%=;\n}" :: "r"(a), "r"(parity) : "memory");
}
__device__ __forceinline__ void tma_box3(uint32_t dst, const CUtensorMap *map, int32_t x, int32_t y, int32_t z,
                                         uint64_t *bar) {
    asm volatile("cp.async.bulk.tensor.3d.shared::cta.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                 :: "r"(dst), "l"(map), "r"(x), "r"(y), "r"(z),
                    "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))) : "memory");
}
__device__ __forceinline__ void tma_gather4(uint32_t dst, const CUtensorMap *map, int32_t x, int32_t r0, int32_t r1,
                                            int32_t r2, int32_t r3, uint64_t *bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 :: "r"(dst), "l"(map), "r"(x), "r"(r0), "r"(r1), "r"(r2), "r"(r3),
                    "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))) : "memory");
}

// Whether (and from which map) unit U stages with TMA: 0 no, 1 A boxes, 2 side boxes,
// 3 gather4.  Its x coordinate (u32 units) comes back in xcoord.
template <int EB, int MODE, int TWB>
__device__ __forceinline__ int tma_kind(const ColParams &P, const Unit &U, uint32_t tt, int32_t &xcoord) {
    if (TWB != 128 || !P.tma || U.skip || U.nslots == 0) return 0;
    const uint32_t mat = fdiv(tt, P.fd_nt);
    const int32_t tile = U.j0 / (TWB / EB);
    if (MODE == COL_R2C_SHUF) {
        if (!(P.tma & 4)) return 0;
        xcoord = U.j0 * EB / 4;
        return 3;
    }
    if (MODE != COL_C2R_SHUF && MODE != COL_ROT) return 0;
    (void)mat;
    // rows wrapping past M - 1, or in the last partial super-row: cp.async
    if (MODE == COL_C2R_SHUF && P.lag == LAG_C2R && tile < P.lagD) {
        if (!(P.tma & 2) || U.rowbase + U.nslots > P.trows_s) return 0;
        xcoord = tile * TWB / 4;
        return 2;
    }
    if (!(P.tma & 1) || U.rowbase + U.nslots > P.trows_a) return 0;
    xcoord = (U.j0 - (MODE == COL_C2R_SHUF && P.lag == LAG_C2R ? P.lagD * (TWB / EB) : 0)) * EB / 4;
    return 1;
}

// Issue the unit's TMA loads (warp 0: lanes split the boxes) and point sbase[] at the 128-byte
// slots.  The caller waits on `bar` (phase `ph`).
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void unit_load_tma(const ColParams &P, const Unit &U, uint32_t tt, int kind, int32_t xcoord,
                                              const int32_t *srow, uint32_t *sbase, uint32_t rows_s, uint64_t *bar) {
    const uint32_t mat = fdiv(tt, P.fd_nt);
    const int lane = threadIdx.x & 31;
    if (kind == 3) {
        for (int32_t t = threadIdx.x; t < U.nslots; t += blockDim.x) sbase[t] = rows_s + static_cast<uint32_t>(t) * TWB;
        if (threadIdx.x >= 32) return;
        const int32_t ng = (U.nslots + 3) / 4;
        if (lane == 0) tmbar_expect(bar, static_cast<uint32_t>(ng) * 4 * TWB);
        __syncwarp();
        const int32_t rbase = static_cast<int32_t>(mat) * P.M;  // packed batch: rows of all matrices
        for (int32_t gi = lane; gi < ng; gi += 32) {
            const int32_t t0 = 4 * gi;
            int32_t r[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) r[e] = rbase + srow[min(t0 + e, U.nslots - 1)];
            tma_gather4(rows_s + static_cast<uint32_t>(t0) * TWB, &P.tmap_g, xcoord, r[0], r[1], r[2], r[3], bar);
        }
    } else {
        // Super-rows of g rows (g = 1 when the pitch is a multiple of 16): slot t (row rowbase
        // + t) has phase p = row mod g; the slots of phase p, t_p, t_p + g, ..., come from the
        // boxes of phase p (x shifted by p rows' worth of bytes, y = super-row) and sit in
        // their own region of whole boxes, R_p.
        const int g = kind == 2 ? P.tg_s : P.tg_a;
        const int64_t pitch = kind == 2 ? P.spitch : static_cast<int64_t>(P.N) * EB;
        int32_t tp[4], reg[4], nbx[4];
        int32_t acc = 0;
#pragma unroll
        for (int p = 0; p < 4; ++p) {
            if (p >= g) break;
            tp[p] = ((p - U.rowbase) % g + g) % g;
            const int32_t np = U.nslots > tp[p] ? (U.nslots - tp[p] + g - 1) / g : 0;
            nbx[p] = (np + kTmaBoxRows - 1) / kTmaBoxRows;
            reg[p] = acc;
            acc += nbx[p] * kTmaBoxRows;
        }
        for (int32_t t = threadIdx.x; t < U.nslots; t += blockDim.x) {
            const int p = (U.rowbase + t) % g;
            sbase[t] = rows_s + static_cast<uint32_t>(reg[p] + (t - tp[p]) / g) * TWB;
        }
        if (threadIdx.x >= 32) return;
        if (lane == 0) tmbar_expect(bar, static_cast<uint32_t>(acc) * TWB);
        __syncwarp();
        const CUtensorMap *map = kind == 2 ? &P.tmap_s : &P.tmap_a;
        for (int p = 0; p < g; ++p) {
            const int32_t x = xcoord + static_cast<int32_t>(p * pitch / 4);
            const int32_t s0 = (U.rowbase + tp[p]) / g;  // first super-row of phase p
            for (int32_t bi = lane; bi < nbx[p]; bi += 32)
                tma_box3(rows_s + static_cast<uint32_t>(reg[p] + bi * kTmaBoxRows) * TWB, map, x, s0 + bi * kTmaBoxRows,
                         static_cast<int32_t>(mat), bar);
        }
    }
}

// Hull staging with 1-D bulk copies (P.bulk; any pitch, not the rightmost tile of a row):
// one cp.async.bulk of a slot's 16-byte-aligned hull (128 or 144 bytes) per lane instead of
// nine 16-byte cp.async; each issuing lane registers its bytes on `bar` (expect_tx), thread 0
// arrives once every lane has issued (the caller's barrier), so the phase cannot complete
// early.  Same slot layout as unit_load (hull pitch, sbase[t] = first tile element).
__device__ __forceinline__ void tmbar_expect_only(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;"
                 :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tmbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];"
                 :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))) : "memory");
}
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void unit_load_bulk(const ColParams &P, const Unit &U, const int32_t *srow, uint32_t *sbase,
                                               uint32_t rows_s, uint64_t *bar) {
    constexpr int HS = hull_pitch(TWB);
    const int64_t pitch = U.in_pitch;
    const uint32_t bar_s = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
    const int32_t tb = U.wt * EB;
    for (int32_t t = threadIdx.x; t < U.nslots; t += blockDim.x) {
        const int32_t g = MODE == COL_R2C_SHUF ? srow[t] : mod_M(U.rowbase + t, P.kshM, P.fd_M);
        const char *rp = U.inp + static_cast<int64_t>(g) * pitch;
        const uint32_t off = static_cast<uint32_t>(reinterpret_cast<uintptr_t>(rp)) & 15u;
        const uint32_t bytes = (off + static_cast<uint32_t>(tb) + 15u) & ~15u;
        const uint32_t dst = rows_s + static_cast<uint32_t>(t) * HS;
        sbase[t] = dst + off;
        tmbar_expect_only(bar, bytes);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(dst), "l"(rp - off), "r"(bytes), "r"(bar_s) : "memory");
    }
}

// Non-persistent variant: one CTA per (tile, band).  The CTA's logical id comes from a
// ticket counter taken at start (dispatch order), so the G members of a tile are exactly
// G consecutive tickets: every group whose tickets are all taken is fully resident, hence
// only the newest group can be waiting for members, and those get scheduled as older
// groups finish.  G == 1: P.tpc consecutive tiles per CTA.
template <int EB, int MODE, int TWB>
__device__ __forceinline__ void col_tile_one(const ColParams &P, unsigned char *smem, uint32_t tt, int32_t r,
                                             uint64_t *tbar, uint32_t &tphase, unsigned int *next_ticket = nullptr) {
    const SmemLayout L = smem_layout(P.B, TWB / EB, TWB, EB);
    int64_t *orow = reinterpret_cast<int64_t *>(smem);
    int32_t *srow = reinterpret_cast<int32_t *>(smem + L.srow);
    uint32_t *sbase = reinterpret_cast<uint32_t *>(smem + L.sbase);
    const Unit U = unit_make<EB, MODE, TWB>(P, tt, r);
    const Dep D = unit_dep<MODE>(P, tt);
    if (U.skip) {  // group-uniform; still arrive, later tiles sharing the counter count it
        if (D.arrive && threadIdx.x == 0) atomicAdd(P.ctr + (tt % kCtrSlots), 1u);
        if (next_ticket && threadIdx.x == 0) *next_ticket = atomicAdd(P.ctr + kTicketSlot, 1u);
        return;
    }
    // R2C: the loads need the scattered source rows (prepass first); otherwise the loads go
    // out first and the C2R destination rows are computed while they are in flight.
    if (MODE == COL_R2C_SHUF) {
        if (P.dbg != 4) unit_prepass<EB, MODE, TWB>(P, U, orow, srow, blockDim.x);
        __syncthreads();
    }
    int32_t xcoord = 0;
    const int kind = tma_kind<EB, MODE, TWB>(P, U, tt, xcoord);
    const uint32_t rows_s = (static_cast<uint32_t>(__cvta_generic_to_shared(smem + L.rows)) + 127u) & ~127u;
    // bulk hulls: not for the rightmost tile of a row (its hull may end past the buffer)
    const bool bulk = !kind && P.bulk && !U.skip && U.j0 + U.wt < P.N && P.dbg != 2;
    if (kind) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // earlier generic reads of the buffer
        unit_load_tma<EB, MODE, TWB>(P, U, tt, kind, xcoord, srow, sbase, rows_s, tbar);
    } else if (bulk) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        unit_load_bulk<EB, MODE, TWB>(P, U, srow, sbase, rows_s, tbar);
    } else if (P.dbg != 2) {  // measurement knob: 2 = skip the loads
        unit_load<EB, MODE, TWB>(P, U, srow, sbase, rows_s, blockDim.x);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    if (MODE != COL_R2C_SHUF && P.dbg != 4) unit_prepass<EB, MODE, TWB>(P, U, orow, srow, blockDim.x);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (bulk) {
        __syncthreads();  // every lane has registered its bytes
        if (threadIdx.x == 0) tmbar_arrive(tbar);
    }
    if (kind || bulk) {
        tmbar_wait(tbar, tphase);
        tphase ^= 1;
    }
    __syncthreads();  // every thread's staged data is in shared memory
    if (threadIdx.x == 0) {
        // The arrival only says "this unit's reads of its input are complete" (write-after-
        // read): every thread's cp.async copies have landed in shared memory (wait_group 0 +
        // the barrier above) before it is issued, so no later write by a waiter can reach
        // them, and a relaxed add suffices.  A release add compiles to MEMBAR.ALL.GPU, which
        // waits on the SM's outstanding stores: 6-8 % of the pass (IPT_COL_DEBUG=7 keeps it).
        if (D.arrive) {
            if (P.dbg == 7)
                asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(P.ctr + (tt % kCtrSlots)) : "memory");
            else
                asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" :: "l"(P.ctr + (tt % kCtrSlots)) : "memory");
        }
        if (D.wait && P.dbg != 5)
            while (!ctr_reached(P, D.on)) __nanosleep(64);
        // persistent grid: the next unit's ticket, taken now so that its latency overlaps
        // the stores (this unit has arrived, so every ticket it could wait for is smaller)
        if (next_ticket) *next_ticket = atomicAdd(P.ctr + kTicketSlot, 1u);
    }
    __syncthreads();
    if (P.dbg == 0 || P.dbg == 7) unit_store<EB, MODE, TWB>(P, U, orow, sbase, blockDim.x);  // 1, 3, 4, 5 = loads only
}

template <int EB, int MODE, int TWB>
__global__ void __launch_bounds__(kColThreads) col_tile_kernel(const __grid_constant__ ColParams P) {
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) uint64_t tbar;  // TMA staging (P.tma)
    uint32_t tphase = 0;
    if (P.tma || P.bulk) {
        if (threadIdx.x == 0) tmbar_init(&tbar);
        __syncthreads();
    }
    // Unit order = dispatch-ticket order (an atomic taken at start).  Barrier mode: a tile's
    // G members are G consecutive dispatches, so the whole group is co-resident.  Lagged
    // layouts only ever wait for units of smaller ticket, which were taken by CTAs already
    // running: no assumption about the order in which the hardware dispatches blocks, or
    // about co-residency with other kernels (MPS, other streams).  P.ticket = 0
    // (IPT_COL_TICKET=0, measurement only) uses the block index instead in lagged mode,
    // which relies on blocks being dispatched in index order.
    __shared__ unsigned int s_ticket;
    unsigned int ticket = blockIdx.x;
    if ((P.lag == LAG_NONE || P.ticket) && P.dbg != 3) {
        if (threadIdx.x == 0) s_ticket = atomicAdd(P.ctr + kTicketSlot, 1u);
        __syncthreads();
        ticket = s_ticket;
    }
    if (P.G == 1) {
        const uint64_t t_end = min(static_cast<uint64_t>(P.total_tiles), (static_cast<uint64_t>(ticket) + 1) * P.tpc);
        for (uint64_t tt = static_cast<uint64_t>(ticket) * P.tpc; tt < t_end; ++tt) {
            col_tile_one<EB, MODE, TWB>(P, smem, static_cast<uint32_t>(tt), 0, &tbar, tphase);
            __syncthreads();  // shared memory is reused by the next tile
        }
        return;
    }
    auto unit_of = [&](unsigned int tk, uint32_t &tt, int32_t &r) {
        if (P.lag != LAG_NONE && P.super > 1) {
            const uint32_t per = static_cast<uint32_t>(P.G) * static_cast<uint32_t>(P.super);
            const uint32_t sidx = tk / per, rem = tk - sidx * per;
            const uint32_t t0 = sidx * static_cast<uint32_t>(P.super);
            const uint32_t here = min(static_cast<uint32_t>(P.super), static_cast<uint32_t>(P.total_tiles) - t0);
            r = static_cast<int32_t>(rem / here);
            tt = t0 + (rem - static_cast<uint32_t>(r) * here);
        } else {
            tt = fdiv(tk, P.fd_G);
            r = static_cast<int32_t>(tk - tt * P.G);
        }
    };
    if (P.persist) {
        // Persistent grid (lagged layouts): resident CTAs loop over tickets, each unit's
        // successor taken during its stores.  Waits still only target smaller tickets, held
        // by running CTAs whose loads wait on nothing (col_tile_one).
        __shared__ unsigned int s_next;
        const uint32_t total = static_cast<uint32_t>(P.total_tiles) * static_cast<uint32_t>(P.G);
        while (ticket < total) {
            uint32_t ptt;
            int32_t pr;
            unit_of(ticket, ptt, pr);
            col_tile_one<EB, MODE, TWB>(P, smem, ptt, pr, &tbar, tphase, &s_next);
            __syncthreads();  // stores done (shared memory reused), s_next published
            ticket = s_next;
        }
        return;
    }
    uint32_t tt;  // tile (of all matrices)
    int32_t r;    // band
    if (P.lag != LAG_NONE && P.super > 1) {
        // super-tile s = tiles [s S, s S + S'), its units band-major: ticket -> (band, tile)
        const uint32_t per = static_cast<uint32_t>(P.G) * static_cast<uint32_t>(P.super);
        const uint32_t s = ticket / per, rem = ticket - s * per;
        const uint32_t t0 = s * static_cast<uint32_t>(P.super);
        const uint32_t here = min(static_cast<uint32_t>(P.super), static_cast<uint32_t>(P.total_tiles) - t0);
        r = static_cast<int32_t>(rem / here);
        tt = t0 + (rem - static_cast<uint32_t>(r) * here);
    } else {
        tt = fdiv(ticket, P.fd_G);
        r = static_cast<int32_t>(ticket - tt * P.G);
    }
    col_tile_one<EB, MODE, TWB>(P, smem, tt, r, &tbar, tphase);
}

// mbarrier helpers (shared::cta).
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))),
                 "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];"
                 :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))) : "memory");
}
// Arrive once every cp.async this thread issued so far has landed (counted in the init).
__device__ __forceinline__ void mbar_arrive_cpasync(uint64_t *bar) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];"
                 :: "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t *bar, unsigned parity) {
    uint32_t ok;
    asm volatile("{\n .reg .pred p;\n mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n"
                 " selp.u32 %0, 1, 0, p;\n}"
                 : "=r"(ok) : "r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar))), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
    asm volatile("{\n .reg .pred p;\n WAIT_%=:\n"
                 " mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], %1;\n"
                 " @!p bra WAIT_%=;\n}" :: "r"(a), "r"(parity) : "memory");
}

// Persistent, warp-specialised, two-buffer variant (P.pipe).  The last two warps are the
// TICKET warp and the CONTROL warp (one thread each), the others are workers.  Unit i of
// a CTA lives in buffer i & 1.  Ticket thread: as soon as unit i-2 is released it takes
// ticket t_i (units in ticket order: tile-major, the G bands of a tile consecutive; the
// atomic's latency overlaps the workers' stores of unit i-2) and publishes it once the
// buffer is free.  Control thread: as soon as the workers' loads of unit i have landed (an
// mbarrier fed by cp.async.mbarrier.arrive) it arrives on the tile's counter --
// independently of how far the older unit has got -- and when the whole group has
// arrived it releases unit i to the workers.  Workers: load unit i, then store unit i-1
// once released.  So the loads of one unit are in flight while the CTA waits for the
// group of the other and stores it, and no group's arrival waits for another group's
// barrier (no lock-step chain).
//
// Deadlock freedom (G <= grid): a unit's arrival needs only its own loads.  Take the
// oldest incomplete group g: its taken tickets all arrive.  If some are untaken, g is the
// newest group (tickets are taken in order); a CTA can take a ticket once a buffer frees,
// and every buffer holding an older unit frees (those groups complete).  Only a CTA whose
// two buffers both hold units of g cannot take more; all CTAs in that state would mean
// >= 2 grid >= G taken tickets of g, i.e. none untaken.  By induction every group completes.
template <int EB, int MODE, int TWB>
__global__ void __launch_bounds__(kColThreads) col_pipe_kernel(const __grid_constant__ ColParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ unsigned int s_ticket[kMaxColBufs];
    __shared__ int s_release;  // units released so far (control -> ticket warp)
    __shared__ __align__(8) uint64_t bar_tk[kMaxColBufs], bar_full[kMaxColBufs], bar_go[kMaxColBufs],
        bar_empty[kMaxColBufs];
    constexpr int W = TWB / EB;
    const int nwt = static_cast<int>(blockDim.x) - 64;  // worker threads
    const int NB = P.nbuf;
    const SmemLayout L = smem_layout(P.B, W, TWB, EB);
    const size_t bufsz = L.total;
    const uint32_t total = static_cast<uint32_t>(P.total_tiles) * static_cast<uint32_t>(P.G);
    if (threadIdx.x == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(&bar_tk[b], 1);
            mbar_init(&bar_full[b], nwt);
            mbar_init(&bar_go[b], 1);
            mbar_init(&bar_empty[b], nwt);
        }
        s_release = 0;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    // Unit u lives in buffer u mod NB and uses phase (u / NB) & 1 of that buffer's mbarriers.

    if (threadIdx.x >= nwt) {
        if (threadIdx.x == nwt) {  // ---- ticket warp: take and publish tickets ----------
            int b = 0, k = 0;
            for (int u = 0;; ++u) {
                if (k > 0) {  // take unit u's ticket once unit u-NB is released: its buffer then
                    // frees unconditionally (the workers only have to store it)
                    while (atomicAdd(&s_release, 0) < u - NB + 1) __nanosleep(32);  // (atomic: no data race)
                }
                const uint32_t t = atomicAdd(P.ctr + kTicketSlot, 1u);
                if (k > 0) mbar_wait(&bar_empty[b], (k - 1) & 1);
                s_ticket[b] = t;
                mbar_arrive(&bar_tk[b]);
                if (t >= total) break;
                if (++b == NB) b = 0, ++k;
            }
        } else if (threadIdx.x == nwt + 32) {  // ---- control warp: arrive and release ----
            int arrive = 0, release = 0;  // next unit to arrive / release
            int ab = 0, ak = 0, rb = 0;
            while (true) {
                bool progress = false;
                if (mbar_test(&bar_tk[ab], ak & 1)) {  // unit `arrive` published
                    const uint32_t t = s_ticket[ab];
                    if (t >= total) {
                        if (release == arrive) break;  // every real unit released
                    } else if (mbar_test(&bar_full[ab], ak & 1)) {
                        const uint32_t tt = fdiv(t, P.fd_G);
                        if (unit_dep<MODE>(P, tt).arrive) group_arrive(P.ctr + (tt % kCtrSlots));
                        ++arrive;
                        if (++ab == NB) ab = 0, ++ak;
                        progress = true;
                    }
                }
                if (release < arrive) {
                    const Dep d = unit_dep<MODE>(P, fdiv(s_ticket[rb], P.fd_G));
                    const bool done = !d.wait || ctr_reached(P, d.on);
                    if (done) {
                        mbar_arrive(&bar_go[rb]);
                        ++release;
                        if (++rb == NB) rb = 0;
                        atomicExch(&s_release, release);
                        progress = true;
                    }
                }
                if (!progress) __nanosleep(32);
            }
        }
        return;
    }

    // ---- workers: load unit i, then store unit i - NB + 1 once released ----------------
    auto store_unit = [&](int sb, int sk) {
        mbar_wait(&bar_go[sb], sk & 1);
        const uint32_t st = s_ticket[sb];
        const uint32_t stt = fdiv(st, P.fd_G);
        const Unit Us = unit_make<EB, MODE, TWB>(P, stt, static_cast<int32_t>(st - stt * P.G));
        unsigned char *sbuf = smem + sb * bufsz;
        unit_store<EB, MODE, TWB>(P, Us, reinterpret_cast<const int64_t *>(sbuf),
                                  reinterpret_cast<const uint32_t *>(sbuf + L.sbase), nwt);
    };
    int b = 0, k = 0;    // buffer / round of unit i
    int sb = 0, sk = 0;  // buffer / round of the oldest unit not yet stored
    for (int i = 0;; ++i) {
        unsigned char *buf = smem + b * bufsz;
        mbar_wait(&bar_tk[b], k & 1);
        const uint32_t t = s_ticket[b];
        if (t >= total) {  // drain: store the units still held, oldest first
            for (int j = max(0, i - NB + 1); j < i; ++j) {
                store_unit(sb, sk);
                if (++sb == NB) sb = 0, ++sk;
            }
            break;
        }
        const uint32_t tt = fdiv(t, P.fd_G);
        const Unit U = unit_make<EB, MODE, TWB>(P, tt, static_cast<int32_t>(t - tt * P.G));
        int64_t *orow = reinterpret_cast<int64_t *>(buf);
        int32_t *srow = reinterpret_cast<int32_t *>(buf + L.srow);
        if (!U.skip) unit_prepass<EB, MODE, TWB>(P, U, orow, srow, nwt);
        asm volatile("bar.sync 1, %0;" :: "r"(nwt) : "memory");  // srow / orow visible
        unit_load<EB, MODE, TWB>(P, U, srow, reinterpret_cast<uint32_t *>(buf + L.sbase),
                                 static_cast<uint32_t>(__cvta_generic_to_shared(buf + L.rows)), nwt);
        mbar_arrive_cpasync(&bar_full[b]);
        if (i - NB + 1 >= 0) {
            store_unit(sb, sk);
            mbar_arrive(&bar_empty[sb]);
            if (++sb == NB) sb = 0, ++sk;
        }
        if (++b == NB) b = 0, ++k;
    }
}

template <int EB, int MODE, int TWB>
void *kptr(bool pipe) {
    return pipe ? reinterpret_cast<void *>(col_pipe_kernel<EB, MODE, TWB>)
                : reinterpret_cast<void *>(col_tile_kernel<EB, MODE, TWB>);
}

template <int EB, int TWB>
void *col_kernel_w(int mode, bool pipe) {
    switch (mode) {
        case COL_ROT: return kptr<EB, COL_ROT, TWB>(pipe);
        case COL_C2R_SHUF: return kptr<EB, COL_C2R_SHUF, TWB>(pipe);
        case COL_R2C_SHUF: return kptr<EB, COL_R2C_SHUF, TWB>(pipe);
        case COL_COPY: return kptr<EB, COL_COPY, TWB>(pipe);
        default: return nullptr;
    }
}

template <int EB>
void *col_kernel_e(int mode, int twb, bool pipe) {
    switch (twb) {
        case 128: return col_kernel_w<EB, 128>(mode, pipe);
        case 256: return col_kernel_w<EB, 256>(mode, pipe);
        case 512: return col_kernel_w<EB, 512>(mode, pipe);
        default: return nullptr;
    }
}

void *col_kernel(int mode, int eb, int twb, bool pipe) {
    switch (eb) {
        case 4: return col_kernel_e<4>(mode, twb, pipe);
        case 8: return col_kernel_e<8>(mode, twb, pipe);
        case 16: return col_kernel_e<16>(mode, twb, pipe);
        default: return nullptr;
    }
}

}  // namespace

size_t col_smem_bytes(int64_t B, int64_t W, int eb, int nbuf) {
    return smem_layout(B, static_cast<int>(W), static_cast<int>(W * eb), eb).total * (nbuf > 0 ? nbuf : 1);
}

int col_max_bufs() { return kMaxColBufs; }

int64_t col_max_band(int64_t W) { return (int64_t(1) << 24) - W; }

int col_block_threads() { return kColThreads; }

int col_resident_ctas(int mode, int eb, int twb, size_t smem, bool pipe, int threads) {
    void *kern = col_kernel(mode, eb, twb, pipe);
    if (!kern || ensure_kernel_attrs(kern, smem, false) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return cached_resident_blocks(kern, threads, smem);
}

cudaError_t launch_col(const ColParams &P0, int mode, int eb, cudaStream_t st, size_t smem) {
    void *kern = col_kernel(mode, eb, P0.W * eb, P0.pipe != 0);
    if (!kern) return cudaErrorInvalidValue;
    cudaError_t e = ensure_kernel_attrs(kern, smem, false);
    if (e != cudaSuccess) return e;
    ColParams P = P0;
    const int64_t units = P.total_tiles * P.G;
    if (units > 0xfffffff0LL) return cudaErrorInvalidConfiguration;
    const int64_t grid = (P.pipe || P.persist) ? std::min<int64_t>(P.resident, units)
                                               : P.G == 1 ? (P.total_tiles + P.tpc - 1) / P.tpc : units;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    // Ticket + group counters: the call's own zeroed scratch (api.cu CallScratch).
    if (!P.ctr) return cudaErrorInvalidValue;
    void *args[] = {&P};
    const int threads = P.threads > 0 ? P.threads : kColThreads;
    // The persistent kernel (barrier mode and IPT_COL_PIPE) runs as a cooperative launch: all
    // of its CTAs (grid <= the co-resident count) are resident at once by construction, which
    // its per-tile group barriers need; a plain launch would only assume it.
    if (P.pipe) return cudaLaunchCooperativeKernel(kern, dim3(static_cast<unsigned>(grid)), dim3(threads), args, smem, st);
    return cudaLaunchKernel(kern, dim3(static_cast<unsigned>(grid)), dim3(threads), args, smem, st);
}

}  // namespace ipt
