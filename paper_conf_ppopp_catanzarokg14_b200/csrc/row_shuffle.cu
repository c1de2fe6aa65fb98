// Row-shuffle kernel (§3 Eq. 24, §4.2 Eq. 31, §4.5 :751).
//
// Every row of the M x N engine view is permuted independently by the same formula
// (Theorem 3: d'_i is a bijection for every i).  B200 realisation of the paper's
// "on-chip row shuffle" (:751): the whole row is staged in shared memory with cp.async
// (16-byte LDGSTS for the aligned interior, element copies for the ragged head/tail --
// rows are 16-byte aligned only when N*eb % 16 == 0), then every warp gathers a
// contiguous segment of the output row from shared memory, lane L writing outputs
// L, L+32, L+64, ... (coalesced stores).  Global traffic: one read and one write of every
// element.
//
// Index forms (Eq. 24 rewritten; derivation in DESIGN.md §"Row shuffle", checked against
// the oracle's Eq. 24 and Eq. 31 by the parity tests).  With j = l b + h (l < c, h < b)
// and f2 = [i + l >= M]:
//   R2C gather  d'_i(j)       = (i + l + h M - M f2) mod N
//   C2R gather  d'^{-1}_i(p)  = l b + (a^{-1} floor(q / c) + f2) mod b,
//               q = (p - i) mod N,  l = q mod c.
// Walking p (or j) in steps of 32 changes the state by per-plan constants plus one carry,
// so a lane spends a handful of integer adds per element (§4.4's strength reduction
// taken one step further); f2 can only be 1 in the last c - 1 rows, which take a
// slower walk that tracks l.
#include <algorithm>
#include <array>
#include <map>
#include <mutex>

#include "plan.h"

namespace ipt {

int row_threads(int64_t N, int eb) { return N * eb >= 48 * 1024 ? 512 : 256; }

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

// C2R walk: src = lb + (hc + f2) mod b with lb = l*b, hc = a^{-1} floor(q/c) mod b.
template <bool TAIL>
struct C2RWalk {
    int32_t lb, hc, l;
    __device__ __forceinline__ C2RWalk(const RowParams &P, int32_t im, int32_t p) {
        int32_t q = p - im;
        q += q < 0 ? P.N : 0;
        const uint32_t col = fdiv(static_cast<uint32_t>(q), P.fd_c);
        l = q - static_cast<int32_t>(col) * P.c;
        lb = l * P.b;
        hc = static_cast<int32_t>(mulmod(static_cast<uint32_t>(P.ainv), col, P.fd_b, P.wide));
    }
    __device__ __forceinline__ int32_t src(const RowParams &P, int32_t Mi) const {
        if (!TAIL) return lb + hc;
        int32_t h = hc + (l >= Mi ? 1 : 0);
        h -= h == P.b ? P.b : 0;
        return lb + h;
    }
    __device__ __forceinline__ void next(const RowParams &P) {
        lb += P.w_dlb;
        const bool carry = lb >= P.N;
        lb -= carry ? P.N : 0;
        hc += P.w_dhc + (carry ? P.ainv : 0);
        hc -= hc >= P.b ? P.b : 0;
        hc -= hc >= P.b ? P.b : 0;
        if (TAIL) {
            l += P.w_dl;
            l -= l >= P.c ? P.c : 0;
        }
    }
};

// R2C walk: src = (i + l + h M) mod N  [- M mod N if f2].
template <bool TAIL>
struct R2CWalk {
    int32_t s, h, l;
    __device__ __forceinline__ R2CWalk(const RowParams &P, int32_t im, int32_t j) {
        l = static_cast<int32_t>(fdiv(static_cast<uint32_t>(j), P.fd_b));
        h = j - l * P.b;
        int32_t t = im + l;
        t -= t >= P.N ? P.N : 0;
        t += static_cast<int32_t>(mulmod(static_cast<uint32_t>(h), static_cast<uint32_t>(P.Mn), P.fd_N, P.wideN));
        t -= t >= P.N ? P.N : 0;
        s = t;
    }
    __device__ __forceinline__ int32_t src(const RowParams &P, int32_t Mi) const {
        if (!TAIL) return s;
        int32_t t = s - (l >= Mi ? P.Mn : 0);
        return t + (t < 0 ? P.N : 0);
    }
    __device__ __forceinline__ void next(const RowParams &P) {
        h += P.w_dh;
        const bool carry = h >= P.b;
        h -= carry ? P.b : 0;
        s += P.w_ds + (carry ? 1 : 0);
        s -= s >= P.N ? P.N : 0;
        if (TAIL) l += P.w_dl2 + (carry ? 1 : 0);
    }
};

// Gather one output row: warps [0, wn) of the row's warp team (this warp is number wl)
// each write a contiguous, 32-aligned segment, lane L writing outputs L, L+32, ...
template <int EB, int DIR, bool TAIL>
__device__ __forceinline__ void gather_row(const RowParams &P, char *row, char *srow, const unsigned char *stage,
                                           int32_t i, int32_t p_begin, int32_t p_end) {
    using T = typename Word<EB>::T;
    const int lane = threadIdx.x & 31;
    const int32_t im = static_cast<int32_t>(fmod_(static_cast<uint32_t>(i), P.fd_N));
    const int32_t Mi = P.M - i;
    const T *src = reinterpret_cast<const T *>(stage);
    // Lagged C2R output (P.shW > 0): logical column p < shW goes to the side row srow, the
    // others to row[p - shW].
    T *out = reinterpret_cast<T *>(row) - P.shW;
    int32_t p = p_begin + lane;
    if (p >= p_end) return;
    if (P.c == 1) {
        // gcd 1 (Theorem 3 with c = 1): the gather index is an arithmetic progression
        // mod N -- C2R d'^{-1}_i(p) = a^{-1} (p - i) mod N, R2C d'_i(j) = (i + j M) mod N --
        // so a lane's next source (32 outputs on) is one add and one conditional subtract.
        uint32_t sidx;
        if (DIR == ROW_C2R) {
            int32_t q = p - im;
            q += q < 0 ? P.N : 0;
            sidx = mulmod(static_cast<uint32_t>(P.ainv), static_cast<uint32_t>(q), P.fd_N, P.wideN);
        } else {
            sidx = static_cast<uint32_t>(im) + mulmod(static_cast<uint32_t>(p), static_cast<uint32_t>(P.Mn), P.fd_N, P.wideN);
            sidx -= sidx >= static_cast<uint32_t>(P.N) ? P.N : 0;
        }
        const uint32_t d = static_cast<uint32_t>(P.c1_step), n = static_cast<uint32_t>(P.N);
        T *o = DIR == ROW_C2R ? out : reinterpret_cast<T *>(row);
        if (DIR == ROW_C2R) {
            const int32_t p_side = min(p_end, P.shW);
            T *so = reinterpret_cast<T *>(srow);
#pragma unroll 4
            for (; p < p_side; p += 32) {
                so[p] = src[sidx];
                sidx += d;
                sidx -= sidx >= n ? n : 0;
            }
        }
#pragma unroll 8
        for (; p < p_end; p += 32) {
            o[p] = src[sidx];
            sidx += d;
            sidx -= sidx >= n ? n : 0;
        }
        return;
    }
    if (DIR == ROW_C2R) {
        C2RWalk<TAIL> w(P, im, p);
        // each lane: its outputs below shW to the side row, then the rest (lanes diverge
        // for at most one iteration; every lane's walk is its own)
        const int32_t p_side = min(p_end, P.shW);
        T *so = reinterpret_cast<T *>(srow);
#pragma unroll 4
        for (; p < p_side; p += 32) {
            so[p] = src[w.src(P, Mi)];
            w.next(P);
        }
#pragma unroll 4
        for (; p < p_end; p += 32) {
            out[p] = src[w.src(P, Mi)];
            w.next(P);
        }
    } else {
        T *o = reinterpret_cast<T *>(row);
        R2CWalk<TAIL> w(P, im, p);
#pragma unroll 4
        for (; p < p_end; p += 32) {
            o[p] = src[w.src(P, Mi)];
            w.next(P);
        }
    }
}

// Bulk prefetch of [p, p + bytes) into L2 (the CTA's threads, 4 KB each).
__device__ __forceinline__ void prefetch_l2(const char *p, int64_t bytes) {
    // cp.async.bulk.prefetch.L2: 16-byte aligned address and size
    const uintptr_t a0 = (reinterpret_cast<uintptr_t>(p) + 15) & ~uintptr_t(15);
    const uintptr_t a1 = (reinterpret_cast<uintptr_t>(p) + bytes) & ~uintptr_t(15);
    for (uintptr_t a = a0 + static_cast<uintptr_t>(threadIdx.x) * 4096; a < a1; a += blockDim.x * 4096ull) {
        const uint32_t sz = a1 - a < 4096 ? static_cast<uint32_t>(a1 - a) : 4096u;
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(a), "r"(sz) : "memory");
    }
}

// Stage one row with cp.async (no commit): smem byte (off + k) holds row byte k, off =
// row & 15.  Whole 16-byte chunks of the row's aligned hull move with 16-byte copies (a
// plain strided loop); the at most two partial chunks at the ends element by element
// (lanes 0.. of warp 0 the head, of warp 1 the tail).
template <int EB>
__device__ __forceinline__ void stage_row_chunks(const char *row, int32_t nbytes, uint32_t sbase) {
    const int off = static_cast<int>(reinterpret_cast<uintptr_t>(row) & 15);  // multiple of EB
    const char *row0 = row - off;
    const int k0 = off ? 1 : 0;                 // first whole chunk
    const int k1 = (off + nbytes) >> 4;         // end of the whole chunks
    for (int k = k0 + threadIdx.x; k < k1; k += blockDim.x) cp_async<16>(sbase + 16 * k, row0 + 16 * k);
    if (EB < 16) {
        const int t = threadIdx.x;
        if (off && t < (16 - off) / EB) {  // head: bytes [0, 16 - off) of the row
            const int q = t * EB;
            if (q < nbytes) cp_async<EB>(sbase + off + q, row + q);
        }
        const int tail = k1 * 16 - off;  // first byte of the partial last chunk
        if (t >= 32 && t - 32 < (nbytes - tail) / EB && tail >= (off ? 16 - off : 0)) {
            const int q = tail + (t - 32) * EB;
            cp_async<EB>(sbase + off + q, row + q);
        }
    }
}

// Stage a lagged R2C input row (P.shW > 0): logical columns [0, shW) from the side row
// `srow`, [shW, N) from row[0, N - shW), so that smem byte (off + k) holds logical byte k,
// off = row & 15 (as stage_row_chunks for an unlagged row).  The side row has the same
// address mod 16 as the row (side_matrix), so both parts move with 16-byte copies.  No commit.
template <int EB>
__device__ __forceinline__ void stage_row_lagged(const RowParams &P, const char *row, const char *srow,
                                                 uint32_t sbase) {
    stage_row_chunks<EB>(srow, P.shW * EB, sbase);
    stage_row_chunks<EB>(row, (P.N - P.shW) * EB, sbase + P.shW * EB);
}

template <int EB>
__device__ __forceinline__ void stage_row(const char *row, int32_t nbytes, uint32_t sbase) {
    stage_row_chunks<EB>(row, nbytes, sbase);
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// Row groups: a CTA stages P.R consecutive rows of one matrix at a time (short rows: one
// row alone keeps too few bytes in flight per SM), and the CTA's warps split into R teams
// of nwarps / R warps, team t gathering row i0 + t.  Group g of the batch is rows
// [i0, i0 + nr) of matrix g / gpm, i0 = (g mod gpm) R, nr = min(R, M - i0).
struct RowGroup {
    int64_t mat;
    int32_t i0, nr;
};
__device__ __forceinline__ RowGroup row_group(const RowParams &P, int64_t g, int32_t gpm) {
    RowGroup G;
    const uint32_t m = fdiv(static_cast<uint32_t>(g), P.fd_gpm);  // groups_total < 2^32 (planner)
    G.mat = m;
    G.i0 = static_cast<int32_t>(static_cast<uint32_t>(g) - m * static_cast<uint32_t>(gpm)) * P.R;
    G.nr = min(P.R, P.M - G.i0);
    return G;
}

// Grid-stride over the row groups.  NBUF = 2: while group g is gathered from one buffer,
// group g + grid is already streaming into the other (cp.async groups), so every CTA
// keeps a group's worth of loads in flight at all times.
template <int EB, int DIR, int NBUF>
__global__ void __launch_bounds__(kRowThreadsMax, 4) row_shuffle_kernel(RowParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int32_t nbytes = P.N * EB;
    const uint32_t rowbuf = (static_cast<uint32_t>(nbytes) + 31) & ~15u;
    const uint32_t bufbytes = rowbuf * static_cast<uint32_t>(P.R);
    const uint32_t sbase = smem_u32(smem);
    const int32_t gpm = (P.M + P.R - 1) / P.R;
    const int64_t groups_total = static_cast<int64_t>(gpm) * P.batch;
    const int wn = (blockDim.x >> 5) / P.R;  // warps per row team
    const int team = (threadIdx.x >> 5) / wn, wl = (threadIdx.x >> 5) - team * wn;
    const int32_t seg = ((P.N + wn - 1) / wn + 31) & ~31;  // output segment of a warp: whole warps' worth
    const int32_t p_begin = wl * seg, p_end = min(P.N, p_begin + seg);
    auto row_ptr = [&](int64_t mm, int32_t ii) {
        return P.base + mm * P.mat_stride_bytes + static_cast<int64_t>(ii) * nbytes;
    };
    auto side_ptr = [&](int64_t mm, int32_t ii) {
        return side_matrix(P.side, P.sstride, mm, P.base + mm * P.mat_stride_bytes) + ii * P.spitch;
    };
    auto stage = [&](const RowGroup &G, int b) {
        for (int32_t rr = 0; rr < G.nr; ++rr) {
            const uint32_t sb = sbase + b * bufbytes + rr * rowbuf;
            if (DIR == ROW_R2C && P.shW) stage_row_lagged<EB>(P, row_ptr(G.mat, G.i0 + rr), side_ptr(G.mat, G.i0 + rr), sb);
            else stage_row_chunks<EB>(row_ptr(G.mat, G.i0 + rr), nbytes, sb);
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    int64_t g = blockIdx.x;
    RowGroup G = row_group(P, g, gpm);
    if (NBUF == 2 && g < groups_total) stage(G, 0);
    int buf = 0;
    for (; g < groups_total; g += gridDim.x) {
        const int64_t ng = g + gridDim.x;
        const RowGroup NG = row_group(P, ng, gpm);
        if (NBUF == 2) {
            if (ng < groups_total) {
                stage(NG, buf ^ 1);
                asm volatile("cp.async.wait_group 1;" ::: "memory");
            } else {
                asm volatile("cp.async.wait_group 0;" ::: "memory");
            }
        } else {
            stage(G, 0);
            // single buffer (rows > 56 KB): the next group streams into L2 meanwhile
            if (ng < groups_total)
                prefetch_l2(row_ptr(NG.mat, NG.i0), static_cast<int64_t>(NG.nr) * nbytes);
            asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        __syncthreads();

        // ---- gather + write back (the last c - 1 rows may have f2 = 1) --------------
        if (team < G.nr) {
            const int32_t i = G.i0 + team;
            char *row = row_ptr(G.mat, i);
            const unsigned char *st = smem + buf * bufbytes + team * rowbuf + (reinterpret_cast<uintptr_t>(row) & 15);
            char *srow = P.shW ? side_ptr(G.mat, i) : nullptr;
            if (i >= P.M - P.c + 1) gather_row<EB, DIR, true>(P, row, srow, st, i, p_begin, p_end);
            else gather_row<EB, DIR, false>(P, row, srow, st, i, p_begin, p_end);
        }
        __syncthreads();  // this buffer is refilled two groups later

        if (NBUF == 2) buf ^= 1;
        G = NG;
    }
}

// ---- Fused rotation + row shuffle (c > 1, c <= kMaxFuseC) --------------------------------
// The engine's column rotation moves column j by rho_j = floor(j/b) in [0, c) rows; for
// small c it folds into the row pass, saving a whole read + write of the matrix.
//  * C2R (Eq. 23 then Eq. 31):  out[i][p] = V_i[d'^{-1}_i(p)],
//        V_i[l] = A[(i + floor(l/b)) mod M][l]  -- the pre-rotated row i,
//    staged as a "staircase": segment rho (source columns [rho b, rho b + b)) comes from row
//    i + rho; rows i + rho >= M come from `wrap`, a copy of rows 0..c-2 taken before the
//    pass.  Each segment sits in its own 16-byte-aligned region at the source's own
//    misalignment, so the interior moves with 16-byte cp.async; padl[rho] maps a source
//    index l to its shared-memory byte (padl[floor(l/b)] + l eb).
//  * R2C (Eq. 24 then Eq. 36):  out[(i + floor(p/b)) mod M][p] = A[i][d'_i(p)]:
//    row i is staged whole and its gathered output block rho is written into row i + rho.
// Rows are processed in groups of P.R consecutive rows (as row_shuffle_kernel).
// In place: flags[row] is set (release) once the row's CTA has read everything it needs.
//  C2R: rows i0.. of a group are written after rows i0-1 .. i0-c+1 (each read a block of a
//  row of the group) are flagged; R2C: a group writes into rows up to i0+nr-1+c-1, after
//  the ones beyond the group are flagged (read by their CTAs).
// No deadlock with a co-resident grid of > c CTAs: every CTA flags its current group before
// it waits, and a waited-for row is either some CTA's current group (flagged) or that CTA's
// later group, which it reaches because its own current group only waits on flagged rows
// (by induction on the chain, whose groups decrease by at least grid - c per hop).
template <int EB>
__device__ __forceinline__ void stage_stair(const RowParams &P, const char *mbase, const char *wrapbase, int32_t i,
                                            uint32_t sbase, int32_t *padl) {
    // Segment rho (source columns [rho b, rho b + b)) of the staircase comes from row i + rho
    // (from `wrap` past the last row); each is staged like a row (stage_row_chunks: 16-byte
    // copies of its aligned hull) into its own region, its byte k at rho segp + so + k.
    const int32_t Lb = P.b * EB;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    for (int32_t rho = 0; rho < P.c; ++rho) {
        const int32_t y = i + rho;
        const char *S = (y < P.M ? mbase + y * pitch : wrapbase + (y - P.M) * pitch) + static_cast<int64_t>(rho) * Lb;
        if (threadIdx.x == 0) padl[rho] = rho * P.segp + static_cast<int32_t>(reinterpret_cast<uintptr_t>(S) & 15) - rho * Lb;
        stage_row_chunks<EB>(S, Lb, sbase + rho * P.segp);
    }
}

// Fused C2R gather of a row with f2 = 0 (i < M - c + 1), vectorised: thread tt of the
// row's team (T threads) writes the 16-byte chunks tt, tt + T, ... of the output row's
// aligned chunk grid (chunk k = logical outputs [k K - oe, k K - oe + K), K = 16 / eb, oe =
// the row's misalignment in elements; the lagged split at shW keeps the alignment, side
// rows being placed like their rows) with one st.global.v4 -- a warp writes 512 contiguous
// bytes -- and the partial chunks (row ends, a chunk straddling shW) element by element.
// Sources: Eq. 31 with q = (p - i) mod N, src = (q mod c) b + (a^{-1} floor(q/c)) mod b,
// stepped by 1 inside a chunk (l += 1; on l == c: l = 0, h += a^{-1}) and by D = T K between
// a thread's chunks (dl = D mod c, dh = a^{-1} floor(D/c) mod b, one carry) -- a few
// integer ops per element instead of a full stride-32 walk per element.
template <int EB>
__device__ __forceinline__ void gather_row_rot_c2r_vec(const RowParams &P, char *mbase, char *srow,
                                                       const unsigned char *buf, const int32_t *padl, int32_t i,
                                                       int32_t tt, int32_t T, int32_t dl, int32_t dh) {
    constexpr int K = 16 / EB;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    char *arow = mbase + static_cast<int64_t>(i) * pitch;
    const int32_t oe = static_cast<int32_t>((reinterpret_cast<uintptr_t>(arow) & 15) / EB);
    const int32_t nk = (P.N + oe + K - 1) / K;
    int32_t k = tt;
    if (k >= nk) return;
    const int32_t im = static_cast<int32_t>(fmod_(static_cast<uint32_t>(i), P.fd_N));
    int32_t q = k * K - oe - im;
    q += q < 0 ? P.N : 0;
    q += q < 0 ? P.N : 0;
    const uint32_t col = fdiv(static_cast<uint32_t>(q), P.fd_c);
    int32_t l = q - static_cast<int32_t>(col) * P.c;
    int32_t h = static_cast<int32_t>(mulmod(static_cast<uint32_t>(P.ainv), col, P.fd_b, P.wide));
    char *sbk = srow;                  // side row (logical p < shW)
    char *abk = arow - P.shW * EB;     // A row (logical p >= shW)
    for (; k < nk; k += T) {
        const int32_t p0 = k * K - oe;
        uint32_t v[4];
        int32_t ll = l, hh = h;
#pragma unroll
        for (int e = 0; e < K; ++e) {
            const uint32_t a = static_cast<uint32_t>(padl[ll] + (ll * P.b + hh) * EB);
            if constexpr (EB == 4) {
                v[e] = *reinterpret_cast<const uint32_t *>(buf + a);
            } else if constexpr (EB == 8) {
                const uint2 x = *reinterpret_cast<const uint2 *>(buf + a);
                v[2 * e] = x.x;
                v[2 * e + 1] = x.y;
            } else {
                const uint4 x = *reinterpret_cast<const uint4 *>(buf + a);
                v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
            }
            if (K > 1) {
                ++ll;
                if (ll == P.c) {
                    ll = 0;
                    hh += P.ainv;
                    hh -= hh >= P.b ? P.b : 0;
                }
            }
        }
        const bool full = p0 >= 0 && p0 + K <= P.N && (p0 >= P.shW || p0 + K <= P.shW);
        if (full) {
            char *dst = (p0 < P.shW ? sbk : abk) + static_cast<int64_t>(p0) * EB;
            stg16(dst, make_uint4(v[0], v[1], v[2], v[3]));
        } else {
#pragma unroll
            for (int e = 0; e < K; ++e) {
                const int32_t p = p0 + e;
                if (p < 0 || p >= P.N) continue;
                char *dst = (p < P.shW ? sbk : abk) + static_cast<int64_t>(p) * EB;
                if constexpr (EB == 4) *reinterpret_cast<uint32_t *>(dst) = v[e];
                else if constexpr (EB == 8) *reinterpret_cast<uint2 *>(dst) = make_uint2(v[2 * e], v[2 * e + 1]);
                else *reinterpret_cast<uint4 *>(dst) = make_uint4(v[0], v[1], v[2], v[3]);
            }
        }
        // next chunk of this thread: q += D
        l += dl;
        const bool carry = l >= P.c;
        l -= carry ? P.c : 0;
        h += dh + (carry ? P.ainv : 0);
        h -= h >= P.b ? P.b : 0;
        h -= h >= P.b ? P.b : 0;
    }
}

template <int EB, int DIR>
__device__ __forceinline__ void gather_row_rot(const RowParams &P, char *mbase, char *srow, const unsigned char *buf,
                                               const int32_t *padl, int32_t i, int32_t p_begin, int32_t p_end) {
    using T = typename Word<EB>::T;
    const int lane = threadIdx.x & 31;
    const int32_t im = static_cast<int32_t>(fmod_(static_cast<uint32_t>(i), P.fd_N));
    const int32_t Mi = P.M - i;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    int32_t p = p_begin + lane;
    if (p >= p_end) return;
    if (DIR == ROW_C2R) {
        // lagged output as in gather_row: p < shW -> side tile row, else row[p - shW]
        T *out = reinterpret_cast<T *>(mbase + static_cast<int64_t>(i) * pitch) - P.shW;
        C2RWalk<true> w(P, im, p);
        const int32_t p_side = min(p_end, P.shW);
        T *so = reinterpret_cast<T *>(srow);
#pragma unroll 4
        for (; p < p_side; p += 32) {
            so[p] = *reinterpret_cast<const T *>(buf + padl[w.l] + w.src(P, Mi) * EB);
            w.next(P);
        }
#pragma unroll 4
        for (; p < p_end; p += 32) {
            out[p] = *reinterpret_cast<const T *>(buf + padl[w.l] + w.src(P, Mi) * EB);
            w.next(P);
        }
    } else {
        const T *src = reinterpret_cast<const T *>(buf);
        R2CWalk<true> w(P, im, p);
        if (i < P.M - P.c + 1) {
            // f2 = 0 in the whole row: the source walk without the f2 term, and the
            // destination (row i + l, column p) as one running pointer that moves by 32
            // columns plus (32 div b + carry) rows per step
            uint32_t sidx = static_cast<uint32_t>(w.s);
            int32_t h = w.h, r = i + w.l;
            r -= r >= P.M ? P.M : 0;
            char *dst = mbase + static_cast<int64_t>(r) * pitch + static_cast<int64_t>(p) * EB;
            const int64_t wrap = static_cast<int64_t>(P.M) * pitch;
            const uint32_t n = static_cast<uint32_t>(P.N);
#pragma unroll 4
            for (; p < p_end; p += 32) {
                *reinterpret_cast<T *>(dst) = src[sidx];
                h += P.w_dh;
                const int32_t carry = h >= P.b ? 1 : 0;
                h -= carry ? P.b : 0;
                sidx += static_cast<uint32_t>(P.w_ds + carry);
                sidx -= sidx >= n ? n : 0;
                const int32_t dl = P.w_dl2 + carry;
                r += dl;
                dst += 32 * EB + static_cast<int64_t>(dl) * pitch;
                if (r >= P.M) {
                    r -= P.M;
                    dst -= wrap;
                }
            }
            return;
        }
#pragma unroll 4
        for (; p < p_end; p += 32) {
            int32_t r = i + w.l;
            r -= r >= P.M ? P.M : 0;
            *reinterpret_cast<T *>(mbase + r * pitch + static_cast<int64_t>(p) * EB) = src[w.src(P, Mi)];
            w.next(P);
        }
    }
}

template <int EB, int DIR, int NBUF>
__global__ void __launch_bounds__(kRowThreadsMax, 4) row_rot_kernel(RowParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t s_cur, s_next;
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    const uint32_t rowbuf = static_cast<uint32_t>(row_fused_smem_bytes(P, EB, DIR));
    const uint32_t bufbytes = rowbuf * static_cast<uint32_t>(P.R);
    const uint32_t padoff = static_cast<uint32_t>(P.c) * static_cast<uint32_t>(P.segp);  // C2R pad table
    const uint32_t sbase = smem_u32(smem);
    const int32_t gpm = (P.M + P.R - 1) / P.R;
    const uint32_t groups_total = static_cast<uint32_t>(gpm) * static_cast<uint32_t>(P.batch);  // < 2^32 (planner)
    const int wn = (blockDim.x >> 5) / P.R;
    const int team = (threadIdx.x >> 5) / wn, wl = (threadIdx.x >> 5) - team * wn;
    const int32_t seg = ((P.N + wn - 1) / wn + 31) & ~31;
    const int32_t p_begin = wl * seg, p_end = min(P.N, p_begin + seg);
    // vectorised C2R gather: the walk constants of a thread's chunk stride D = 32 wn 16 / eb
    const int64_t vD = static_cast<int64_t>(wn) * 32 * (16 / EB);
    const int32_t vdl = static_cast<int32_t>(vD % P.c);
    const int32_t vdh = static_cast<int32_t>((static_cast<int64_t>(P.ainv) * ((vD / P.c) % P.b)) % P.b);

    // Work order.  Groups are handed out by a dispatch ticket (an atomic), C2R in ascending
    // row order, R2C in descending row order within each matrix, so that every row a group
    // waits for (C2R: rows i0-1 .. i0-c+1; R2C: rows i0+nr .. i0+nr+c-2 < M) belongs to a
    // group with a SMALLER ticket -- one already taken by a running CTA.  The rows whose
    // readers would otherwise come later (C2R: staircases past row M-1; R2C: writes of the
    // last rows' blocks into rows 0..c-2) read the wrap copy of rows 0..c-2 instead, taken
    // before this pass.  Progress (no co-residency assumption, no dispatch-order assumption):
    // a group is flagged once it is staged and its CTA's previous group has been gathered; a
    // gather waits only for flags of smaller tickets; by induction on the ticket, the
    // smallest unflagged group gets flagged.
    auto group_of = [&](uint32_t t) {
        const uint32_t mat = fdiv(t, P.fd_gpm);
        uint32_t gm = t - mat * static_cast<uint32_t>(gpm);
        if (DIR == ROW_R2C) gm = static_cast<uint32_t>(gpm) - 1 - gm;
        RowGroup G;
        G.mat = mat;
        G.i0 = static_cast<int32_t>(gm) * P.R;
        G.nr = min(P.R, P.M - G.i0);
        return G;
    };
    auto a_row = [&](const RowGroup &G, char *mb, int32_t i) -> const char * {
        // R2C: rows 0..c-2 from their wrap copy (same address mod 16 as the row)
        if (DIR == ROW_R2C && i < P.c - 1) return wrap_matrix(P.wrap, P.wstride, G.mat, mb) + i * pitch;
        return mb + i * pitch;
    };
    auto stage = [&](const RowGroup &G, int b) {
        char *mb = P.base + G.mat * P.mat_stride_bytes;
        for (int32_t rr = 0; rr < G.nr; ++rr) {
            const uint32_t o = b * bufbytes + rr * rowbuf;
            const int32_t i = G.i0 + rr;
            if (DIR == ROW_C2R)
                stage_stair<EB>(P, mb, wrap_matrix(P.wrap, P.wstride, G.mat, mb), i, sbase + o,
                                reinterpret_cast<int32_t *>(smem + o + padoff));
            else if (P.shW)
                stage_row_lagged<EB>(P, a_row(G, mb, i), side_matrix(P.side, P.sstride, G.mat, mb) + i * P.spitch,
                                     sbase + o);
            else
                stage_row_chunks<EB>(a_row(G, mb, i), P.N * EB, sbase + o);
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    // The group's reads are complete (after cp.async.wait_group 0 and a __syncthreads): the
    // flag only orders those completed reads before the neighbours' writes (write-after-
    // read), so a relaxed store suffices -- a release store is a MEMBAR.ALL.GPU, which waits
    // on the SM's outstanding stores (as col_tile.cu's arrivals).
    auto set_flags = [&](const RowGroup &G) {
        if (threadIdx.x < G.nr)
            asm volatile("st.relaxed.gpu.global.u32 [%0], %1;"
                         :: "l"(P.flags + G.mat * P.M + G.i0 + threadIdx.x), "r"(1u) : "memory");
    };
    auto wait_deps = [&](const RowGroup &G) {  // every row the group overwrites has been read
        if (threadIdx.x >= 1 && threadIdx.x < P.c) {
            const int32_t y = DIR == ROW_C2R ? G.i0 - static_cast<int32_t>(threadIdx.x)
                                             : G.i0 + G.nr - 1 + static_cast<int32_t>(threadIdx.x);
            if (y >= 0 && y < P.M) {
                const unsigned int *f = P.flags + G.mat * P.M + y;
                unsigned int v;
                while (true) {
                    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(f) : "memory");
                    if (v) break;
                    __nanosleep(32);
                }
            }
        }
        __syncthreads();
    };
    if (threadIdx.x == 0) {
        s_cur = atomicAdd(P.ticket, 1u);
        s_next = s_cur < groups_total ? atomicAdd(P.ticket, 1u) : groups_total;
    }
    __syncthreads();
    uint32_t tc = s_cur, tn = s_next;
    if (tc >= groups_total) return;
    // NBUF = 2: the next group is staged while the current one is gathered, and flagged as
    // soon as the gather of the current group is done -- a full group ahead of the moment
    // its neighbours wait.  The ticket after it is taken during the gather.
    RowGroup G = group_of(tc);
    stage(G, 0);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncthreads();
    set_flags(G);
    int buf = 0;
    while (tc < groups_total) {
        char *mbase = P.base + G.mat * P.mat_stride_bytes;
        const bool more = tn < groups_total;
        const RowGroup NG = more ? group_of(tn) : G;
        if (NBUF == 2 && more) stage(NG, buf ^ 1);
        if (NBUF == 1 && more)  // single buffer: the next group's rows stream into L2 meanwhile
            prefetch_l2(P.base + NG.mat * P.mat_stride_bytes + NG.i0 * pitch, static_cast<int64_t>(NG.nr) * pitch);
        wait_deps(G);
        if (threadIdx.x == 0 && more) s_next = atomicAdd(P.ticket, 1u);  // published by the barrier below

        if (team < G.nr) {
            const int32_t i = G.i0 + team;
            const unsigned char *b = smem + buf * bufbytes + team * rowbuf;
            char *srow = P.shW ? side_matrix(P.side, P.sstride, G.mat, mbase) + i * P.spitch : nullptr;
            if (DIR == ROW_C2R) {
                if (P.vec && i < P.M - P.c + 1)
                    gather_row_rot_c2r_vec<EB>(P, mbase, srow, b, reinterpret_cast<const int32_t *>(b + padoff), i,
                                               wl * 32 + (threadIdx.x & 31), wn * 32, vdl, vdh);
                else
                    gather_row_rot<EB, DIR>(P, mbase, srow, b, reinterpret_cast<const int32_t *>(b + padoff), i,
                                            p_begin, p_end);
            } else {
                gather_row_rot<EB, DIR>(P, mbase, srow, b + (reinterpret_cast<uintptr_t>(mbase + i * pitch) & 15),
                                        nullptr, i, p_begin, p_end);
            }
        }
        if (NBUF == 2) {
            // one barrier: this buffer is free again AND the prefetched group has landed
            asm volatile("cp.async.wait_group 0;" ::: "memory");
            __syncthreads();
            if (more) set_flags(NG);
        } else {
            __syncthreads();  // this buffer is free again
            if (more) {
                stage(NG, 0);
                asm volatile("cp.async.wait_group 0;" ::: "memory");
                __syncthreads();
                set_flags(NG);
            }
        }
        if (NBUF == 2) buf ^= 1;
        tc = tn;
        G = NG;
        tn = more ? s_next : groups_total;
    }
}

// Copy rows 0..c-2 of every matrix of the batch into its wrap slot (wrap_matrix: same address
// mod 16 as the rows, so the body moves with 16-byte accesses; every offset is a multiple of 4).
__global__ void __launch_bounds__(256) copy_wrap_kernel(char *base, int64_t mat_stride, int64_t batch, char *wrap,
                                                        int64_t wstride, int64_t bytes) {
    for (int64_t mat = blockIdx.y; mat < batch; mat += gridDim.y) {
        const char *src = base + mat * mat_stride;
        char *dst = wrap_matrix(wrap, wstride, mat, src);
        const int64_t mis = static_cast<int64_t>((16 - (reinterpret_cast<uintptr_t>(src) & 15)) & 15);
        const int64_t head = bytes < mis ? bytes : mis;
        const int64_t body = (bytes - head) & ~int64_t(15);
        const int64_t tid = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
        const int64_t nth = static_cast<int64_t>(gridDim.x) * blockDim.x;
        for (int64_t k = tid; k < body / 16; k += nth)
            stg16(dst + head + 16 * k, ldg16(src + head + 16 * k));
        if (tid < head / 4)
            reinterpret_cast<uint32_t *>(dst)[tid] = reinterpret_cast<const uint32_t *>(src)[tid];
        const int64_t t0 = head + body;
        if (tid < (bytes - t0) / 4)
            reinterpret_cast<uint32_t *>(dst + t0)[tid] = reinterpret_cast<const uint32_t *>(src + t0)[tid];
    }
}

// ---- Cluster row pass (rows longer than one CTA's shared memory) -----
// A cluster of K CTAs owns one row at a time.  CTA k stages row elements
// [k seg, (k+1) seg) in its shared memory; after a cluster barrier every CTA gathers its
// own output segment, reading each source element from the shared memory of the CTA that
// holds it (ld.shared::cluster, distributed shared memory), and writes it coalesced.  A
// second barrier (the loop's) keeps a CTA's buffer alive until every peer has read it.
// In place: all global reads of a row precede the barrier, all its writes follow it.
__device__ __forceinline__ uint32_t mapa_u32(uint32_t a, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
    return r;
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// cluster_barrier() (arrive.release / wait.acquire) compiles to MEMBAR.ALL.GPU, which
// waits for every outstanding global store of the thread.  This form orders the thread's
// prior accesses at CTA scope only (MEMBAR.ALL.CTA) -- IPT_ROW_CLUSTER_SYNC selects it.
__device__ __forceinline__ void cluster_barrier_cta_fence() {
    asm volatile("fence.acq_rel.cta;\n"
                 "barrier.cluster.arrive.relaxed.aligned;\n"
                 "barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
}
template <int EB>
__device__ __forceinline__ typename Word<EB>::T ld_cluster(uint32_t a) {
    typename Word<EB>::T v;
    // volatile keeps these loads between the cluster barriers; no "memory" clobber, so
    // the global stores of the gather may be scheduled after a batch of loads
    if constexpr (EB == 4) {
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a));
    } else if constexpr (EB == 8) {
        asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(v) : "r"(a));
    } else {
        asm volatile("ld.shared::cluster.v4.u32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    }
    return v;
}

template <int EB, int DIR, bool TAIL>
__device__ __forceinline__ void gather_seg(const RowParams &P, char *row, uint32_t rb, int32_t p0, int32_t p1,
                                           int32_t i) {
    using T = typename Word<EB>::T;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    const int32_t len = p1 - p0;
    const int32_t per = ((len + nwarps - 1) / nwarps + 31) & ~31;
    const int32_t p_end = min(p1, p0 + warp * per + per);
    const int32_t im = static_cast<int32_t>(fmod_(static_cast<uint32_t>(i), P.fd_N));
    const int32_t Mi = P.M - i;
    T *out = reinterpret_cast<T *>(row);
    int32_t p = p0 + warp * per + lane;
    if (p - lane >= p_end) return;  // warp-uniform
    // lane k < K holds the cluster address of CTA k's staged segment (rb)
    auto fetch = [&](int32_t s) {
        const uint32_t owner = fdiv(static_cast<uint32_t>(s), P.fd_seg);
        const uint32_t base = __shfl_sync(0xffffffffu, rb, static_cast<int>(owner));
        return ld_cluster<EB>(base + static_cast<uint32_t>(s - static_cast<int32_t>(owner) * P.cl_seg) * EB);
    };
    // __shfl_sync needs the whole warp: lanes past the end keep walking without storing.
    // Batches of U remote loads are issued before their stores (memory-level parallelism:
    // a distributed-shared-memory load costs a round trip through the cluster network).
    constexpr int U = 8;
    auto run = [&](auto w) {
        for (; p - lane < p_end; p += 32 * U) {
            T v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                v[u] = fetch(w.src(P, Mi));
                w.next(P);
            }
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (p + 32 * u < p_end) out[p + 32 * u] = v[u];
        }
    };
    if (DIR == ROW_C2R) run(C2RWalk<TAIL>(P, im, min(p, P.N - 1)));
    else run(R2CWalk<TAIL>(P, im, min(p, P.N - 1)));
}

template <int EB, int DIR>
__global__ void __launch_bounds__(kRowThreadsMax) row_cluster_kernel(RowParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    const uint32_t K = static_cast<uint32_t>(P.cl_K);
    const uint32_t rank = cluster_rank();
    const int64_t cid = blockIdx.x / K, ncl = gridDim.x / K;
    const int64_t rows_total = static_cast<int64_t>(P.M) * P.batch;
    const int32_t nbytes = P.N * EB;
    const uint32_t sbase = smem_u32(smem);
    const int lane = threadIdx.x & 31;
    const uint32_t rb0 = lane < static_cast<int>(K) ? mapa_u32(sbase, static_cast<uint32_t>(lane)) : 0;
    const int32_t p0 = static_cast<int32_t>(rank) * P.cl_seg;
    const int32_t p1 = min(P.N, p0 + P.cl_seg);
    for (int64_t r = cid; r < rows_total; r += ncl) {
        const int64_t mat = r / P.M;
        const int32_t i = static_cast<int32_t>(r - mat * P.M);
        char *row = P.base + mat * P.mat_stride_bytes + static_cast<int64_t>(i) * nbytes;
        if (p1 > p0) {
            stage_row<EB>(row + static_cast<int64_t>(p0) * EB, (p1 - p0) * EB, sbase);
            asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        // every segment of the row is staged and visible cluster-wide
        if (P.cl_sync >= 2) cluster_barrier_cta_fence();
        else cluster_barrier();
        // seg * EB is a multiple of 16: all segments share the row's 16-byte misalignment
        const uint32_t rb = rb0 + static_cast<uint32_t>(reinterpret_cast<uintptr_t>(row) & 15);
        if (p1 > p0) {
            if (i >= P.M - P.c + 1) gather_seg<EB, DIR, true>(P, row, rb, p0, p1, i);
            else gather_seg<EB, DIR, false>(P, row, rb, p0, p1, i);
        }
        // peers are done reading this CTA's buffer (a WAR hazard only: the reads have
        // returned -- their values feed the stores issued before the arrive)
        if (P.cl_sync >= 1) cluster_barrier_cta_fence();
        else cluster_barrier();
    }
}

// L2 variant (cl_mode 1): CTA k gathers its output segment [k seg, (k+1) seg) straight from
// the row in global memory (random reads served by L2; the row is prefetched into L2 one
// row ahead with bulk prefetches) into its shared memory; one cluster barrier (every read
// of the row is done) and the segment is written back coalesced.  Shared memory is private
// to the CTA, so one barrier per row suffices.
template <int EB, int DIR, bool TAIL>
__device__ __forceinline__ void gather_l2(const RowParams &P, const char *row, const char *srow, unsigned char *buf,
                                          int32_t p0, int32_t p1, int32_t i) {
    using T = typename Word<EB>::T;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    const int32_t len = p1 - p0;
    const int32_t per = ((len + nwarps - 1) / nwarps + 31) & ~31;
    const int32_t p_end = min(p1, p0 + warp * per + per);
    const int32_t im = static_cast<int32_t>(fmod_(static_cast<uint32_t>(i), P.fd_N));
    const int32_t Mi = P.M - i;
    // Lagged R2C input (P.shW > 0): logical element s < shW in the side row, else row[s - shW].
    const T *src = reinterpret_cast<const T *>(row) - (DIR == ROW_R2C ? P.shW : 0);
    const T *ssrc = reinterpret_cast<const T *>(srow);
    T *out = reinterpret_cast<T *>(buf) - p0;
    int32_t p = p0 + warp * per + lane;
    if (p >= p_end) return;
    constexpr int U = 8;
    auto run = [&](auto w) {
        for (; p < p_end; p += 32 * U) {
            T v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int32_t s = w.src(P, Mi);
                if (p + 32 * u < p_end) v[u] = __ldcg((DIR == ROW_R2C && s < P.shW ? ssrc : src) + s);
                w.next(P);
            }
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (p + 32 * u < p_end) out[p + 32 * u] = v[u];
        }
    };
    if (DIR == ROW_C2R) run(C2RWalk<TAIL>(P, im, p));
    else run(R2CWalk<TAIL>(P, im, p));
}


template <int EB, int DIR>
__global__ void __launch_bounds__(kRowThreadsMax) row_cluster_l2_kernel(RowParams P) {
    using T = typename Word<EB>::T;
    extern __shared__ __align__(16) unsigned char smem[];
    const uint32_t K = static_cast<uint32_t>(P.cl_K);
    const uint32_t rank = cluster_rank();
    const int64_t cid = blockIdx.x / K, ncl = gridDim.x / K;
    const int64_t rows_total = static_cast<int64_t>(P.M) * P.batch;
    const int32_t nbytes = P.N * EB;
    const int32_t p0 = static_cast<int32_t>(rank) * P.cl_seg;
    const int32_t p1 = min(P.N, p0 + P.cl_seg);
    auto row_of = [&](int64_t r) {
        const int64_t mat = r / P.M;
        return P.base + mat * P.mat_stride_bytes + static_cast<int64_t>(r - mat * P.M) * nbytes;
    };
    // Lagged layouts (P.shW > 0, shared with the column pass): R2C reads logical columns
    // [0, shW) from the side row and [shW, N) from row[0, N - shW); C2R writes them there.
    auto side_of = [&](int64_t r) -> char * {
        if (!P.shW) return nullptr;
        const int64_t mat = r / P.M;
        return side_matrix(P.side, P.sstride, mat, P.base + mat * P.mat_stride_bytes) + (r - mat * P.M) * P.spitch;
    };
    // this CTA's share of the row's L2 prefetch (segment [p0, p1) of the row, its side part too)
    auto prefetch = [&](int64_t r) {
        if (p1 <= p0) return;
        prefetch_l2(row_of(r) + static_cast<int64_t>(p0) * EB, (p1 - p0) * EB);
        if (DIR == ROW_R2C && P.shW && p0 < P.shW) prefetch_l2(side_of(r) + static_cast<int64_t>(p0) * EB,
                                                             (min(p1, P.shW) - p0) * EB);
    };
    if (cid < rows_total) prefetch(cid);
    for (int64_t r = cid; r < rows_total; r += ncl) {
        const int32_t i = static_cast<int32_t>(r % P.M);
        char *row = row_of(r);
        char *srow = side_of(r);
        if (r + ncl < rows_total) prefetch(r + ncl);
        if (p1 > p0) {
            if (i >= P.M - P.c + 1) gather_l2<EB, DIR, true>(P, row, srow, smem, p0, p1, i);
            else gather_l2<EB, DIR, false>(P, row, srow, smem, p0, p1, i);
        }
        // every CTA of the cluster has read the whole row (its loads have returned)
        cluster_barrier_cta_fence();
        const T *buf = reinterpret_cast<const T *>(smem);
        if (DIR == ROW_C2R && P.shW) {
            T *dst = reinterpret_cast<T *>(row) - P.shW;
            T *sdst = reinterpret_cast<T *>(srow);
            for (int32_t k = threadIdx.x; k < p1 - p0; k += blockDim.x) {
                const int32_t pp = p0 + k;
                (pp < P.shW ? sdst : dst)[pp] = buf[k];
            }
        } else {
            T *dst = reinterpret_cast<T *>(row) + p0;
            for (int32_t k = threadIdx.x; k < p1 - p0; k += blockDim.x) dst[k] = buf[k];
        }
        __syncthreads();  // the buffer is refilled by the next row
    }
}

template <int EB, int DIR>
cudaError_t launch_row_cluster_t(const RowParams &P, cudaStream_t st, int active_only, int *active) {
    const size_t smem = row_cluster_smem(P.cl_seg, EB);
    auto kern = P.cl_mode == 1 ? row_cluster_l2_kernel<EB, DIR> : row_cluster_kernel<EB, DIR>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, P.cl_K > 8);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg{};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = static_cast<unsigned>(P.cl_K);
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cfg.blockDim = dim3(kRowThreadsMax);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    if (active_only) {
        int sms = 0, dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cfg.gridDim = dim3(static_cast<unsigned>(sms / P.cl_K * P.cl_K));
        return cudaOccupancyMaxActiveClusters(active, reinterpret_cast<const void *>(kern), &cfg);
    }
    const int64_t rows = static_cast<int64_t>(P.M) * P.batch;
    int64_t ncl = *active;
    if (ncl > rows) ncl = rows;
    cfg.gridDim = dim3(static_cast<unsigned>(ncl * P.cl_K));
    e = cudaLaunchKernelEx(&cfg, kern, P);
    return e != cudaSuccess ? e : cudaGetLastError();
}

template <int EB>
cudaError_t launch_row_cluster_e(const RowParams &P, int dir, cudaStream_t st, int active_only, int *active) {
    return dir == ROW_C2R ? launch_row_cluster_t<EB, ROW_C2R>(P, st, active_only, active)
                          : launch_row_cluster_t<EB, ROW_R2C>(P, st, active_only, active);
}

cudaError_t row_cluster_dispatch(const RowParams &P, int dir, int eb, cudaStream_t st, int active_only, int *active) {
    switch (eb) {
        case 4: return launch_row_cluster_e<4>(P, dir, st, active_only, active);
        case 8: return launch_row_cluster_e<8>(P, dir, st, active_only, active);
        case 16: return launch_row_cluster_e<16>(P, dir, st, active_only, active);
        default: return cudaErrorInvalidValue;
    }
}



// ---- Warp-specialised row pass (default; IPT_ROW_PIPE=0 keeps the kernels above) ------
// One PRODUCER warp stages row groups with TMA bulk copies (cp.async.bulk, one per row part:
// the 16-byte-aligned interior; the at most 3 + 3 words of ragged head / tail with 4-byte
// cp.async) into NBUF mbarrier-tracked buffers; NW CONSUMER warps gather and write the
// rows.  full[b]: 32 arrivals (every producer lane, once its small copies have landed and its
// pad-table entries are written) + the bulk bytes; empty[b]: one arrival per consumer
// thread once it no longer reads the
// buffer, and the producer fences the generic proxy against the async one before it
// refills a buffer.  Every thread orders its own accesses with its own arrive / wait.  No
// CTA-wide barrier on the data path: warps run ahead / behind independently.  Same shared-
// memory layout as row_shuffle_kernel, so the gather (gather_row) is shared; the chunked
// fused pass below uses the same structure.
__device__ __forceinline__ void pmbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void pmbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" :: "r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void pmbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" :: "r"(bar) : "memory");
}
__device__ __forceinline__ void pmbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile("{\n .reg .pred p;\n WAIT_%=:\n"
                 " mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], %1;\n"
                 " @!p bra WAIT_%=;\n}" :: "r"(bar), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}

// Stage one contiguous part of a row: global bytes [gs, gs + nb) land at shared byte
// sd16 + (x - floor16(gs)) (sd16 16-byte aligned).  Interior by one bulk copy (expect_tx
// first), ragged ends word by word with 4-byte cp.async (every offset is a multiple of 4).
__device__ __forceinline__ void stage_part(const char *gs, int32_t nb, uint32_t sd16, uint32_t bar) {
    if (nb <= 0) return;
    const uintptr_t g = reinterpret_cast<uintptr_t>(gs);
    const uintptr_t g16 = g & ~uintptr_t(15);
    const uintptr_t a0 = (g + 15) & ~uintptr_t(15), a1 = (g + nb) & ~uintptr_t(15);
    auto word = [&](uintptr_t x) {
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(sd16 + static_cast<uint32_t>(x - g16)),
                     "l"(reinterpret_cast<const void *>(x)) : "memory");
    };
    if (a1 > a0) {
        const uint32_t bytes = static_cast<uint32_t>(a1 - a0);
        pmbar_expect_tx(bar, bytes);
        bulk_g2s(sd16 + static_cast<uint32_t>(a0 - g16), reinterpret_cast<const void *>(a0), bytes, bar);
        for (uintptr_t x = g; x < a0; x += 4) word(x);
        for (uintptr_t x = a1; x < g + nb; x += 4) word(x);
    } else {
        for (uintptr_t x = g; x < g + nb; x += 4) word(x);
    }
}

template <int EB, int DIR, int NBUF, int NW>
__global__ void __launch_bounds__(NW * 32 + 32, NW == 16 ? 2 : 4) row_pipe_kernel(RowParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ __align__(8) uint64_t bar_full[NBUF], bar_empty[NBUF];
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    const uint32_t rowbuf = static_cast<uint32_t>((static_cast<uint32_t>(P.N) * EB + 31) & ~15u);
    const uint32_t bufbytes = rowbuf * static_cast<uint32_t>(P.R);
    const uint32_t sbase = smem_u32(smem);
    const int32_t gpm = (P.M + P.R - 1) / P.R;
    const uint32_t groups_total = static_cast<uint32_t>(gpm) * static_cast<uint32_t>(P.batch);  // < 2^32 (planner)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int b = 0; b < NBUF; ++b) {
            pmbar_init(smem_u32(&bar_full[b]), 32);
            pmbar_init(smem_u32(&bar_empty[b]), NW * 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (P.zero && blockIdx.x == 0)
        for (int32_t k = threadIdx.x; k < P.zero_words; k += blockDim.x) P.zero[k] = 0u;
    // Row groups in grid-stride order: CTA blockIdx.x takes groups blockIdx.x + k gridDim.x
    // (producer and consumers walk the same sequence).
    auto mat_base = [&](const RowGroup &G) { return P.base + G.mat * P.mat_stride_bytes; };

    if (warp == NW) {
        // ================================ producer ================================
        uint32_t t = blockIdx.x;
        for (uint32_t k = 0; t < groups_total; ++k, t += gridDim.x) {
            const int b = static_cast<int>(k % NBUF);
            const uint32_t fb = smem_u32(&bar_full[b]);
            if (k >= NBUF) {
                pmbar_wait(smem_u32(&bar_empty[b]), ((k / NBUF) - 1) & 1);
                // the consumers' generic-proxy reads of this buffer before the bulk copies'
                // async-proxy writes into it
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            }
            const RowGroup G = row_group(P, t, gpm);
            char *mb = mat_base(G);
            const uint32_t sb0 = sbase + b * bufbytes;
            // whole rows; lagged R2C rows in two parts (side row, row), both at the row's alignment
            const int parts = (DIR == ROW_R2C && P.shW) ? 2 : 1;
            for (int32_t pi = lane; pi < G.nr * parts; pi += 32) {
                const int32_t rr = pi / parts, part = pi - rr * parts;
                const int32_t i = G.i0 + rr;
                const char *row = mb + i * pitch;
                const uint32_t reg = sb0 + rr * rowbuf;
                if (parts == 1) {
                    stage_part(row, P.N * EB, reg, fb);
                } else if (part == 0) {
                    stage_part(side_matrix(P.side, P.sstride, G.mat, mb) + i * P.spitch, P.shW * EB, reg, fb);
                } else {
                    stage_part(row, (P.N - P.shW) * EB, reg + P.shW * EB, fb);
                }
            }
            __syncwarp();
            // every lane: its small copies have landed and its pad-table entries are written
            asm volatile("cp.async.wait_all;" ::: "memory");
            pmbar_arrive(fb);
            const uint32_t tn = t + gridDim.x;
            if (NBUF == 1 && tn < groups_total && lane == 0) {
                // single buffer: the next group's rows stream into L2 while this one is gathered
                const RowGroup NG = row_group(P, tn, gpm);
                const char *a = mat_base(NG) + NG.i0 * pitch;
                const uintptr_t a0 = (reinterpret_cast<uintptr_t>(a) + 15) & ~uintptr_t(15);
                const uintptr_t a1 = (reinterpret_cast<uintptr_t>(a) + NG.nr * pitch) & ~uintptr_t(15);
                for (uintptr_t x = a0; x < a1; x += 32768) {
                    const uint32_t sz = a1 - x < 32768 ? static_cast<uint32_t>(a1 - x) : 32768u;
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(x), "r"(sz) : "memory");
                }
            }
        }
        return;
    }

    // ================================ consumers ================================
    const int wn = NW / P.R;  // warps per row team
    const int team = warp / wn, wl = warp - team * wn;
    const int32_t seg = ((P.N + wn - 1) / wn + 31) & ~31;
    const int32_t p_begin = wl * seg, p_end = min(P.N, p_begin + seg);
    uint32_t t = blockIdx.x;
    for (uint32_t k = 0; t < groups_total; ++k, t += gridDim.x) {
        const int b = static_cast<int>(k % NBUF);
        pmbar_wait(smem_u32(&bar_full[b]), (k / NBUF) & 1);
        const RowGroup G = row_group(P, t, gpm);
        char *mbase = mat_base(G);
        if (team < G.nr) {
            const int32_t i = G.i0 + team;
            const unsigned char *buf = smem + b * bufbytes + team * rowbuf;
            char *row = mbase + i * pitch;
            const unsigned char *st = buf + (reinterpret_cast<uintptr_t>(row) & 15);
            char *srow = P.shW ? side_matrix(P.side, P.sstride, G.mat, mbase) + i * P.spitch : nullptr;
            if (i >= P.M - P.c + 1) gather_row<EB, DIR, true>(P, row, srow, st, i, p_begin, p_end);
            else gather_row<EB, DIR, false>(P, row, srow, st, i, p_begin, p_end);
        }
        pmbar_arrive(smem_u32(&bar_empty[b]));  // every lane: its reads of the buffer are done
    }
}

// ---- Chunked fused rotation + row pass (default for 1 < c <= kMaxFuseC) ---------------
// Same producer / consumer structure and staging as row_pipe_kernel, but the work unit
// is a CHUNK of cK consecutive rows of one matrix, whose row groups a CTA processes in order:
//  * C2R (Eq. 23 then Eq. 31): writing row i overwrites segments that only the staircases of
//    rows i-c+1 .. i read; those of the same chunk were staged (landed) before row i's group
//    is gathered (the consumer takes groups in order), those of the previous chunk read the
//    boundary copy of this chunk's first c-1 rows instead.
//  * R2C (Eq. 24 then Eq. 36), descending: row i's blocks go to rows i .. i+c-1, staged
//    earlier in the chunk; rows of the next chunk (or rows 0..c-2 past row M-1) are read by
//    their own chunk from its boundary copy.
// So no CTA waits for another: no flags, no tickets, no co-residency assumption.  Extra
// traffic: the boundary copy, 2 (c-1) / cK of a pass.
template <int EB, int DIR, int NBUF, int NW>
__global__ void __launch_bounds__(NW * 32 + 32, NW == 16 ? 2 : 4) row_chunk_kernel(RowParams P) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ __align__(8) uint64_t bar_full[NBUF], bar_empty[NBUF];
    const int64_t pitch = static_cast<int64_t>(P.N) * EB;
    const uint32_t rowbuf = static_cast<uint32_t>(row_fused_smem_bytes(P, EB, DIR));
    const uint32_t bufbytes = rowbuf * static_cast<uint32_t>(P.R);
    const uint32_t padoff = static_cast<uint32_t>(P.c) * static_cast<uint32_t>(P.segp);  // C2R pad table
    const uint32_t sbase = smem_u32(smem);
    const int64_t total_chunks = static_cast<int64_t>(P.nch) * P.batch;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int b = 0; b < NBUF; ++b) {
            pmbar_init(smem_u32(&bar_full[b]), 32);
            pmbar_init(smem_u32(&bar_empty[b]), NW * 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (P.zero && blockIdx.x == 0)
        for (int32_t k = threadIdx.x; k < P.zero_words; k += blockDim.x) P.zero[k] = 0u;
    // The (chunk, group) sequence of this CTA -- walked identically by producer and consumers.
    struct Seq {
        int64_t ch, mat;
        int32_t x, r0, r1, ng, gi;
    };
    auto chunk_at = [&](Seq &q, int64_t ch) {
        q.ch = ch;
        if (ch >= total_chunks) return false;
        q.mat = static_cast<int64_t>(fdiv(static_cast<uint32_t>(ch), P.fd_nch));  // total_chunks < 2^32
        q.x = static_cast<int32_t>(ch - q.mat * P.nch);
        q.r0 = q.x * P.cK;
        q.r1 = min(P.M, q.r0 + P.cK);
        q.ng = (q.r1 - q.r0 + P.R - 1) / P.R;
        q.gi = 0;
        return true;
    };
    auto advance = [&](Seq &q) {  // next group; false at the end of this CTA's work
        if (++q.gi < q.ng) return true;
        return chunk_at(q, q.ch + gridDim.x);
    };
    auto group_of = [&](const Seq &q) {
        RowGroup G;
        G.mat = q.mat;
        const int32_t g = DIR == ROW_C2R ? q.gi : q.ng - 1 - q.gi;
        G.i0 = q.r0 + g * P.R;
        G.nr = min(P.R, q.r1 - G.i0);
        return G;
    };
    auto mat_base = [&](int64_t mat) { return P.base + mat * P.mat_stride_bytes; };

    if (warp == NW) {
        // ================================ producer ================================
        Seq q;
        bool more = chunk_at(q, blockIdx.x);
        for (uint32_t k = 0; more; ++k) {
            const int b = static_cast<int>(k % NBUF);
            const uint32_t fb = smem_u32(&bar_full[b]);
            if (k >= NBUF) {
                pmbar_wait(smem_u32(&bar_empty[b]), ((k / NBUF) - 1) & 1);
                // the consumers' generic-proxy reads of this buffer before the bulk copies'
                // async-proxy writes into it
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            }
            const RowGroup G = group_of(q);
            char *mb = mat_base(G.mat);
            const uint32_t sb0 = sbase + b * bufbytes;
            if (DIR == ROW_C2R) {
                // staircase: segment rho of row i = source columns [rho b, rho b + b) of row
                // i + rho -- from the boundary copy of the next chunk (chunk 0 past row M-1)
                const int32_t Lb = P.b * EB;
                for (int32_t pi = lane; pi < G.nr * P.c; pi += 32) {
                    const int32_t rr = pi / P.c, rho = pi - rr * P.c;
                    const int32_t y = G.i0 + rr + rho;
                    const char *rowp;
                    if (y < q.r1) {
                        rowp = mb + y * pitch;
                    } else if (y < P.M) {
                        rowp = bnd_row(P.bnd, P.rpitch, P.nch, P.c, G.mat, q.x + 1, y - q.r1, mb + y * pitch);
                    } else {
                        rowp = bnd_row(P.bnd, P.rpitch, P.nch, P.c, G.mat, 0, y - P.M, mb + (y - P.M) * pitch);
                    }
                    const char *S = rowp + static_cast<int64_t>(rho) * Lb;
                    const uint32_t reg = sb0 + rr * rowbuf + rho * P.segp;
                    int32_t *padl = reinterpret_cast<int32_t *>(smem + b * bufbytes + rr * rowbuf + padoff);
                    padl[rho] = rho * P.segp + static_cast<int32_t>(reinterpret_cast<uintptr_t>(S) & 15) - rho * Lb;
                    stage_part(S, Lb, reg, fb);
                }
            } else {
                // whole rows, the chunk's first c-1 from its boundary copy; lagged rows in two
                // parts (side row, row), both at the row's alignment
                const int parts = P.shW ? 2 : 1;
                for (int32_t pi = lane; pi < G.nr * parts; pi += 32) {
                    const int32_t rr = pi / parts, part = pi - rr * parts;
                    const int32_t i = G.i0 + rr;
                    const char *row = i - q.r0 < P.c - 1
                                          ? bnd_row(P.bnd, P.rpitch, P.nch, P.c, G.mat, q.x, i - q.r0, mb + i * pitch)
                                          : mb + i * pitch;
                    const uint32_t reg = sb0 + rr * rowbuf;
                    if (parts == 1) {
                        stage_part(row, P.N * EB, reg, fb);
                    } else if (part == 0) {
                        stage_part(side_matrix(P.side, P.sstride, G.mat, mb) + i * P.spitch, P.shW * EB, reg, fb);
                    } else {
                        stage_part(row, (P.N - P.shW) * EB, reg + P.shW * EB, fb);
                    }
                }
            }
            __syncwarp();
            // every lane: its small copies have landed and its pad-table entries are written
            asm volatile("cp.async.wait_all;" ::: "memory");
            pmbar_arrive(fb);
            more = advance(q);
            if (NBUF == 1 && more && lane == 0) {
                // single buffer: the next group's rows stream into L2 while this one is gathered
                const RowGroup NG = group_of(q);
                const char *a = mat_base(NG.mat) + NG.i0 * pitch;
                const uintptr_t a0 = (reinterpret_cast<uintptr_t>(a) + 15) & ~uintptr_t(15);
                const uintptr_t a1 = (reinterpret_cast<uintptr_t>(a) + NG.nr * pitch) & ~uintptr_t(15);
                for (uintptr_t xx = a0; xx < a1; xx += 32768) {
                    const uint32_t sz = a1 - xx < 32768 ? static_cast<uint32_t>(a1 - xx) : 32768u;
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(xx), "r"(sz) : "memory");
                }
            }
        }
        return;
    }

    // ================================ consumers ================================
    const int wn = NW / P.R;  // warps per row team
    const int team = warp / wn, wl = warp - team * wn;
    const int32_t seg = ((P.N + wn - 1) / wn + 31) & ~31;
    const int32_t p_begin = wl * seg, p_end = min(P.N, p_begin + seg);
    const int64_t vD = static_cast<int64_t>(wn) * 32 * (16 / EB);
    const int32_t vdl = static_cast<int32_t>(vD % P.c);
    const int32_t vdh = static_cast<int32_t>((static_cast<int64_t>(P.ainv) * ((vD / P.c) % P.b)) % P.b);
    Seq q;
    bool more = chunk_at(q, blockIdx.x);
    for (uint32_t k = 0; more; ++k) {
        const int b = static_cast<int>(k % NBUF);
        pmbar_wait(smem_u32(&bar_full[b]), (k / NBUF) & 1);
        const RowGroup G = group_of(q);
        char *mbase = mat_base(G.mat);
        if (team < G.nr) {
            const int32_t i = G.i0 + team;
            const unsigned char *buf = smem + b * bufbytes + team * rowbuf;
            char *srow = P.shW ? side_matrix(P.side, P.sstride, G.mat, mbase) + i * P.spitch : nullptr;
            if (DIR == ROW_C2R) {
                if (P.vec && i < P.M - P.c + 1)
                    gather_row_rot_c2r_vec<EB>(P, mbase, srow, buf, reinterpret_cast<const int32_t *>(buf + padoff), i,
                                               wl * 32 + lane, wn * 32, vdl, vdh);
                else
                    gather_row_rot<EB, DIR>(P, mbase, srow, buf, reinterpret_cast<const int32_t *>(buf + padoff), i,
                                            p_begin, p_end);
            } else {
                gather_row_rot<EB, DIR>(P, mbase, srow, buf + (reinterpret_cast<uintptr_t>(mbase + i * pitch) & 15),
                                        nullptr, i, p_begin, p_end);
            }
        }
        pmbar_arrive(smem_u32(&bar_empty[b]));  // every lane: its reads of the buffer are done
        more = advance(q);
    }
}

// Boundary copy of the chunked fused pass: rows [x cK, x cK + c - 1) (clamped to M) of every
// chunk x of every matrix into bnd_row() slots; one CTA per (matrix, chunk), threads over the
// row's 16-byte chunks (same address mod 16 on both sides; every offset is a multiple of 4).
__global__ void __launch_bounds__(256) copy_bounds_kernel(RowParams P, int64_t pitch) {
    const int64_t slots = static_cast<int64_t>(P.nch) * P.batch;
    for (int64_t sl = blockIdx.x; sl < slots; sl += gridDim.x) {
        const int64_t mat = sl / P.nch;
        const int32_t x = static_cast<int32_t>(sl - mat * P.nch);
        const int32_t r0 = x * P.cK, nr = min(P.c - 1, P.M - r0);
        char *mb = P.base + mat * P.mat_stride_bytes;
        for (int32_t r = 0; r < nr; ++r) {
            const char *src = mb + (r0 + r) * pitch;
            char *dst = bnd_row(P.bnd, P.rpitch, P.nch, P.c, mat, x, r, src);
            const int64_t mis = static_cast<int64_t>((16 - (reinterpret_cast<uintptr_t>(src) & 15)) & 15);
            const int64_t head = pitch < mis ? pitch : mis;
            const int64_t body = (pitch - head) & ~int64_t(15);
            for (int64_t kk = threadIdx.x; kk < body / 16; kk += blockDim.x)
                stg16(dst + head + 16 * kk, ldg16(src + head + 16 * kk));
            if (threadIdx.x < head / 4)
                reinterpret_cast<uint32_t *>(dst)[threadIdx.x] = reinterpret_cast<const uint32_t *>(src)[threadIdx.x];
            const int64_t t0 = head + body;
            if (threadIdx.x < (pitch - t0) / 4)
                reinterpret_cast<uint32_t *>(dst + t0)[threadIdx.x] = reinterpret_cast<const uint32_t *>(src + t0)[threadIdx.x];
        }
    }
}

template <int EB, int DIR, int NBUF, int NW>
cudaError_t launch_row_chunk_t(const RowParams &P, cudaStream_t st) {
    const size_t smem = NBUF * P.R * row_fused_smem_bytes(P, EB, DIR);
    auto kern = row_chunk_kernel<EB, DIR, NBUF, NW>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int threads = NW * 32 + 32;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), threads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    if (!P.bnd) return cudaErrorInvalidValue;
    const int64_t chunks = static_cast<int64_t>(P.nch) * P.batch;
    int64_t grid = resident;
    if (grid > chunks) grid = chunks;
    kern<<<static_cast<unsigned>(grid), threads, smem, st>>>(P);
    return cudaGetLastError();
}

template <int EB, int DIR, int NBUF>
cudaError_t launch_row_chunk_n(const RowParams &P, cudaStream_t st) {
    return row_threads(P.N, EB) == 512 ? launch_row_chunk_t<EB, DIR, NBUF, 16>(P, st)
                                       : launch_row_chunk_t<EB, DIR, NBUF, 8>(P, st);
}

template <int EB, int DIR, int NBUF, int NW>
cudaError_t launch_row_pipe_t(const RowParams &P, cudaStream_t st) {
    const size_t smem = NBUF * P.R * row_smem_bytes(P.N, EB);
    auto kern = row_pipe_kernel<EB, DIR, NBUF, NW>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int threads = NW * 32 + 32;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), threads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t groups = static_cast<int64_t>((P.M + P.R - 1) / P.R) * P.batch;
    int64_t grid = resident;
    if (grid > groups) grid = groups;
    kern<<<static_cast<unsigned>(grid), threads, smem, st>>>(P);
    return cudaGetLastError();
}

template <int EB, int DIR, int NBUF>
cudaError_t launch_row_pipe_n(const RowParams &P, cudaStream_t st) {
    return row_threads(P.N, EB) == 512 ? launch_row_pipe_t<EB, DIR, NBUF, 16>(P, st)
                                       : launch_row_pipe_t<EB, DIR, NBUF, 8>(P, st);
}

template <int EB, int DIR, int NBUF>
cudaError_t launch_row_t(const RowParams &P, cudaStream_t st) {
    const size_t smem = NBUF * P.R * row_smem_bytes(P.N, EB);
    const int threads = row_threads(P.N, EB);
    auto kern = row_shuffle_kernel<EB, DIR, NBUF>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), threads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t rows = static_cast<int64_t>((P.M + P.R - 1) / P.R) * P.batch;
    int64_t grid = resident;
    if (grid > rows) grid = rows;
    kern<<<static_cast<unsigned>(grid), threads, smem, st>>>(P);
    return cudaGetLastError();
}

template <int EB, int DIR, int NBUF>
cudaError_t launch_row_rot_t(const RowParams &P, cudaStream_t st) {
    const size_t smem = NBUF * P.R * row_fused_smem_bytes(P, EB, DIR);
    const int threads = row_threads(P.N, EB);
    auto kern = row_rot_kernel<EB, DIR, NBUF>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), threads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    if (!P.ticket || !P.flags || !P.wrap) return cudaErrorInvalidValue;
    const int64_t rows = static_cast<int64_t>((P.M + P.R - 1) / P.R) * P.batch;
    int64_t grid = resident;
    if (grid > rows) grid = rows;
    kern<<<static_cast<unsigned>(grid), threads, smem, st>>>(P);
    return cudaGetLastError();
}

template <int EB, int DIR>
cudaError_t launch_row_d(const RowParams &P, cudaStream_t st) {
    if (P.fuse && P.chunk)
        return 2 * P.R * row_fused_smem_bytes(P, EB, DIR) <= static_cast<size_t>(P.db_max)
                   ? launch_row_chunk_n<EB, DIR, 2>(P, st)
                   : launch_row_chunk_n<EB, DIR, 1>(P, st);
    if (P.pipe && !P.fuse)
        return 2 * P.R * row_smem_bytes(P.N, EB) <= static_cast<size_t>(P.db_max)
                   ? launch_row_pipe_n<EB, DIR, 2>(P, st)
                   : launch_row_pipe_n<EB, DIR, 1>(P, st);
    if (P.fuse)
        return 2 * P.R * row_fused_smem_bytes(P, EB, DIR) <= static_cast<size_t>(P.db_max)
                   ? launch_row_rot_t<EB, DIR, 2>(P, st)
                                                                         : launch_row_rot_t<EB, DIR, 1>(P, st);
    return 2 * P.R * row_smem_bytes(P.N, EB) <= static_cast<size_t>(P.db_max) ? launch_row_t<EB, DIR, 2>(P, st)
                                                           : launch_row_t<EB, DIR, 1>(P, st);
}

}  // namespace

cudaError_t launch_copy_wrap(const RowParams &P, int eb, cudaStream_t st) {
    (void)eb;
    const int64_t bytes = static_cast<int64_t>(P.c - 1) * P.N * eb;
    if (bytes <= 0) return cudaSuccess;
    const int64_t chunks = (bytes + 16 * 256 - 1) / (16 * 256);
    const unsigned gx = static_cast<unsigned>(std::min<int64_t>(chunks, 64));
    const unsigned gy = static_cast<unsigned>(std::min<int64_t>(P.batch, 65535));
    copy_wrap_kernel<<<dim3(gx, gy), 256, 0, st>>>(P.base, P.mat_stride_bytes, P.batch, P.wrap, P.wstride, bytes);
    return cudaGetLastError();
}

cudaError_t launch_copy_bounds(const RowParams &P, int eb, cudaStream_t st) {
    const int64_t slots = static_cast<int64_t>(P.nch) * P.batch;
    if (P.c <= 1 || slots <= 0) return cudaSuccess;
    const unsigned grid = static_cast<unsigned>(std::min<int64_t>(slots, 4096));
    copy_bounds_kernel<<<grid, 256, 0, st>>>(P, static_cast<int64_t>(P.N) * eb);
    return cudaGetLastError();
}

size_t row_smem_bytes(int64_t N, int eb) { return (static_cast<size_t>(N) * eb + 31) & ~size_t(15); }
int row_block_threads() { return kRowThreadsMax; }

size_t row_cluster_smem(int32_t seg, int eb) { return static_cast<size_t>(seg) * eb + 32; }

int row_cluster_active(int K, int32_t seg, int eb, int dir, int mode) {
    static std::mutex mu;
    static std::map<std::array<int, 6>, int> cache;
    int dev = 0;
    cudaGetDevice(&dev);
    const std::array<int, 6> key{K, seg, eb, dir, dev, mode};
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find(key);
        if (it != cache.end()) return it->second;
    }
    RowParams P{};
    P.cl_K = K;
    P.cl_seg = seg;
    P.cl_mode = mode;
    int active = 0;
    if (row_cluster_dispatch(P, dir, eb, nullptr, 1, &active) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    std::lock_guard<std::mutex> lk(mu);
    cache[key] = active;
    return active;
}

cudaError_t launch_row_cluster(const RowParams &P, int dir, int eb, cudaStream_t st) {
    int active = row_cluster_active(P.cl_K, P.cl_seg, eb, dir, P.cl_mode);
    if (active < 1) return cudaErrorInvalidConfiguration;
    return row_cluster_dispatch(P, dir, eb, st, 0, &active);
}

cudaError_t launch_row(const RowParams &P, int dir, int eb, cudaStream_t st) {
    switch (eb * 2 + dir) {
        case 4 * 2 + ROW_C2R: return launch_row_d<4, ROW_C2R>(P, st);
        case 4 * 2 + ROW_R2C: return launch_row_d<4, ROW_R2C>(P, st);
        case 8 * 2 + ROW_C2R: return launch_row_d<8, ROW_C2R>(P, st);
        case 8 * 2 + ROW_R2C: return launch_row_d<8, ROW_R2C>(P, st);
        case 16 * 2 + ROW_C2R: return launch_row_d<16, ROW_C2R>(P, st);
        case 16 * 2 + ROW_R2C: return launch_row_d<16, ROW_R2C>(P, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace ipt
