// Host planner and kernel parameter blocks of the CUDA path.
//
// An engine works on the buffer viewed as an M x N row-major array (rows of N contiguous
// elements).  c = gcd(M, N), a = M / c, b = N / c.
//   C2R(M, N) realises P_{M,N} ("transpose the row-major M x N buffer", Theorem 1):
//       [column rotation r_j, Eq. 23, if c > 1] -> row gather d'^{-1}_i (Eq. 31)
//       -> column gather s'_j = p_j o q (Eqs. 26, 32, 33)
//   R2C(M, N) realises P_{N,M} = P_{M,N}^{-1} (§4.3):
//       column gather q^{-1}((i - j) mod M) (Eqs. 34, 35) -> row gather d'_i (Eq. 24)
//       -> [column rotation r^{-1}_j, Eq. 36, if c > 1]
#pragma once

#include <cstddef>
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

#include "common.cuh"

namespace ipt {

enum Engine : int { ENG_NONE = 0, ENG_C2R = 1, ENG_R2C = 2, ENG_SKINNY = 3 };

// Column-tile kernel modes.
enum ColMode : int {
    COL_ROT = 0,       // out[i][j] = in[(i + sign*floor(j/b)) mod M][j]   (Eq. 23 / Eq. 36)
    COL_C2R_SHUF = 1,  // out[i][j] = in[(j + q(i)) mod M][j]              (Eq. 26 = p_j o q)
    COL_R2C_SHUF = 2,  // out[i][j] = in[q^{-1}((i - j) mod M)][j]         (Eqs. 34, 35)
    COL_COPY = 3,      // out[i][j] = in[i][j]: measurement of the tile access pattern only
                       // (ipt_debug_tile_copy); rot_sign = 0 also drops the cluster barrier
};

// Column-shuffle tile layouts (col_tile.cu, "In-place hazard").
enum ColLag : int { LAG_NONE = 0, LAG_R2C = 1, LAG_C2R = 2 };
// Side tiles of the lagged layouts: matrix k's M x (D W) side block, rows spitch bytes apart,
// placed so that side row i has the same address mod 16 as row i of the matrix (spitch =
// N eb mod 16): the lagged row pass stages side part and row part with 16-byte copies.
__host__ __device__ inline char *side_matrix(char *side, int64_t sstride, int64_t mat, const char *A_mat) {
    char *raw = side + mat * sstride;
    return raw + ((reinterpret_cast<uintptr_t>(A_mat) - reinterpret_cast<uintptr_t>(raw)) & 15);
}
// Wrap rows of the fused rotation: matrix k's copy of rows 0..c-2, placed so that copy row i
// has the same address mod 16 as row i of the matrix (staged with the same 16-byte copies).
__host__ __device__ inline char *wrap_matrix(char *wrap, int64_t wstride, int64_t mat, const char *A_mat) {
    char *raw = wrap + mat * wstride;
    return raw + ((reinterpret_cast<uintptr_t>(A_mat) - reinterpret_cast<uintptr_t>(raw)) & 15);
}
// Boundary row r (< c-1) of chunk x of matrix `mat` (chunked fused pass), placed at the same
// address mod 16 as the matrix row it copies (A_row), so it stages like that row.
__host__ __device__ inline char *bnd_row(char *bnd, int64_t rpitch, int64_t nch, int32_t c, int64_t mat, int64_t x,
                                         int32_t r, const char *A_row) {
    char *raw = bnd + ((mat * nch + x) * (c - 1) + r) * rpitch;
    return raw + ((reinterpret_cast<uintptr_t>(A_row) - reinterpret_cast<uintptr_t>(raw)) & 15);
}
// Row-shuffle directions.
enum RowDir : int {
    ROW_C2R = 0,  // out[i][j] = in[i][d'^{-1}_i(j)]  (Eq. 31)
    ROW_R2C = 1,  // out[i][j] = in[i][d'_i(j)]       (Eq. 24 as a gather, §4.3 :717)
};

struct RowParams {
    char *base;
    int64_t mat_stride_bytes;  // distance between matrices of a batch
    int64_t batch;
    int32_t M, N, c, a, b;
    int32_t ainv;   // mmi(a, b)
    int32_t amodb;  // a mod b
    int32_t Mn;     // M mod N
    FastDiv fd_c, fd_b, fd_N;
    int32_t wide;   // b >= 2^16: products need 64 bits
    int32_t wideN;  // N >= 2^16
    // Per-plan constants of a 32-element stride along the row (row_shuffle.cu walks):
    int32_t w_dl;   // 32 mod c
    int32_t w_dlb;  // (32 mod c) * b
    int32_t w_dhc;  // a^{-1} floor(32 / c) mod b
    int32_t w_dh;   // 32 mod b
    int32_t w_dl2;  // floor(32 / b)
    int32_t w_ds;   // (floor(32 / b) + (32 mod b) M) mod N
    int32_t c1_step;  // c = 1: the gather index step of 32 outputs, (32 a^{-1}) mod N (C2R) or
                      // (32 M) mod N (R2C)
    // Cluster row pass (rows too long for one CTA): the row is split
    // into cl_K segments of cl_seg elements (a multiple of 32), one per CTA of a cluster.
    int32_t cl_K, cl_seg;
    int32_t cl_sync;  // 0: release/acquire cluster barriers; 1: CTA fence before the WAR
                      // barrier; 2: CTA fences on both (IPT_ROW_CLUSTER_SYNC)
    int32_t cl_mode;  // 0: stage the row across the cluster, gather through DSMEM;
                      // 1: gather from the row in L2 into private shared memory
                      // (IPT_ROW_CLUSTER_MODE)
    FastDiv fd_seg;
    // Fused rotation (c > 1, c <= kMaxFuseC; row_rot_kernel): the column rotation of the
    // engine (C2R pre-rotation Eq. 23 / R2C post-rotation Eq. 36) folded into this pass.
    int32_t fuse;
    int32_t vec;             // fused C2R: vectorised gather for rows with f2 = 0 (IPT_ROW_VEC)
    int32_t R;               // rows per CTA stage (row groups; a power of two dividing the warps)
    int32_t db_max;          // double-buffer the row stage while two buffers fit in this many bytes
    int32_t pipe;            // 1: warp-specialised pass (bulk-copy producer warp, row_pipe_kernel)
    FastDiv fd_gpm;          // ceil(M / R): row groups per matrix
    // Lagged layout shared with the column shuffle (col_tile.cu): logical columns [0, shW)
    // of row i live in the side tile, side + (mat M + i) spitch; columns [shW, N) at A
    // columns [0, N - shW).  R2C reads it (the column pass ran first), C2R writes it.
    int32_t shW;
    int64_t spitch, sstride;  // as ColParams (side_matrix)
    char *side;
    int32_t segp;            // C2R staircase: shared bytes per source segment (b elements)
    FastDiv fd_cps;          // segp / 16 (16-byte chunks per segment)
    unsigned int *flags;     // per-row "read" flags (M * batch, zeroed per call)
    unsigned int *ticket;    // row-group dispatch ticket of the fused pass (zeroed per call)
    char *wrap;              // copy of rows 0..c-2 of every matrix (wrap_matrix(); taken before
                             // the fused pass: C2R staircases past row M-1 read it, R2C reads
                             // rows 0..c-2 from it so that writes into them need no wait)
    int64_t wstride;         // bytes reserved per matrix in `wrap`
    // Chunked fused pass (row_chunk_kernel, default for the fused rotation): every matrix
    // is cut into nch chunks of cK consecutive rows; a CTA processes a chunk's row groups in
    // order (C2R ascending, R2C descending).  The first c-1 rows of every chunk are copied to
    // `bnd` before the pass (launch_copy_bounds): C2R staircases that cross into the next
    // chunk (or past row M-1: chunk 0) and R2C reads of a chunk's own first rows use the copy,
    // so no CTA ever waits for another.
    int32_t chunk;           // 1: chunked fused pass
    int32_t cK, nch;         // rows per chunk (a multiple of R), chunks per matrix
    FastDiv fd_nch;
    char *bnd;               // boundary rows: bnd_row()
    int64_t rpitch;          // bytes per boundary row slot (N eb rounded up to 16, + 16)
    // C2R calls whose first pass is this row pass: CTA 0 zeroes the column pass's counters
    // (zero_words words at `zero`), which saves the call's memset (api.cu launch_call).
    unsigned int *zero;
    int32_t zero_words;
};
constexpr int kMaxFuseC = 32;

// TMA staging of the column pass: 2-D tiles of kTmaBoxRows rows x 128 bytes (A and side
// block, 3-D maps over the batch; any pitch, via super-rows) and R2C row gathers of 4 rows
// (tile::gather4, a 2-D map over all rows, 16-byte pitches; batches packed only).
constexpr int kTmaBoxRows = 16;
struct ColParams {
    CUtensorMap tmap_a;   // 3-D {N eb / 4, M, batch} u32, box {32, kTmaBoxRows, 1}
    CUtensorMap tmap_s;   // 3-D {spitch / 4, M, batch} u32 over the side block (lagged C2R input)
    CUtensorMap tmap_g;   // 2-D {N eb / 4, M batch} u32, box {32, 1} (gather4)
    int32_t tma;          // bit 0: box loads of A; bit 1: box loads of the side block; bit 2: gather4
    // Super-rows: rows of a pitch that is not a multiple of 16 bytes are grouped g at a time
    // (g = 16 / gcd(pitch, 16)), so that the map's row pitch g pitch is; a box at x = (phase
    // pitch + column bytes) / 4 then loads every g-th row of one phase.  Rows of whole
    // super-rows only (trows = g floor(M / g)).
    int32_t tg_a, tg_s, trows_a, trows_s;
    char *base;
    int64_t mat_stride_bytes;
    int64_t batch;
    int32_t M, N, c, a, b;
    int32_t binv;   // mmi(b, a)
    FastDiv fd_c, fd_a, fd_b, fd_M;
    int32_t W, log2W;   // tile width in elements (power of two)
    int32_t ntiles;     // ceil(N / W) tiles per matrix
    int32_t G;          // CTAs per group = bands per tile: ceil(M / B)
    int32_t B;          // rows per CTA band
    int32_t ngroups;    // groups in the persistent grid (grid = ngroups * G)
    int32_t resident;   // co-resident CTAs of this configuration (SMs x CTAs per SM)
    int64_t total_tiles;  // ntiles * batch
    unsigned int *ctr;  // arrival counters + dispatch ticket: kCtrSlots + 1 words of the call's
                        // stream-ordered scratch, zeroed before the launch (api.cu CallScratch)
    int32_t ticket;     // 1: units in dispatch-ticket order (an atomic per CTA); 0: block index
    int32_t persist;    // lagged layouts, G > 1: persistent grid of resident CTAs looping over tickets
    int32_t bulk;       // hull staging with one 1-D bulk copy per slot (instead of 16-byte cp.async)
    int32_t super;      // lagged layouts: units ordered band-major within super-tiles of `super`
                        // consecutive tiles (<= lagD), so that concurrently running units read
                        // adjacent 128-byte segments of the same rows (1: tile-major)
    int32_t rot_sign;   // COL_ROT: +1 (C2R pre-rotation) or -1 (R2C post-rotation)
    int32_t wide_a;     // a >= 2^16
    FastDiv fd_G, fd_nt;  // ticket -> (tile, band), tile -> (matrix, column tile)
    uint32_t kshM;      // (2 + W / M) * M: shift making every mod_M argument non-negative
    int32_t tpc;        // tiles per CTA when G == 1 (each tile fits one CTA)
    int32_t pipe;       // 1: persistent pipelined kernel (col_pipe_kernel) with nbuf unit buffers
    int32_t nbuf;
    int32_t threads;    // threads per CTA (col_block_threads() for the pipelined kernel)
    int32_t lag;        // LAG_NONE, LAG_R2C or LAG_C2R (col_tile.cu: lagged tile layouts)
    char *side;         // LAG_*: the side tiles (side_matrix() locates a matrix's)
    int32_t lagD;       // LAG_*: the lag in tiles (tiles 0..D-1 live in the side tiles)
    int64_t spitch;     // side row pitch: D TWB + (N eb mod 16) (rows as aligned as A's)
    int64_t sstride;    // side bytes reserved per matrix
    int32_t dbg;        // measurement only (IPT_COL_DEBUG): 1 loads only, 3 + no ticket, 4 + no prepass,
                        // 5 loads only without the wait, 7 release arrivals
};

// Skinny engine storage: "location" L in [0, n] is row L of the n x N view, location n is
// the one-row buffer tmp.  Logical row r's column block rho = floor(j / b) lives at
// the location below between the passes (rolling rows with the rotation folded in, DESIGN.md
// §"Skinny engine"):
//   R2C (AoS -> SoA): column pass writes (r, rho) to  r == n-1 ? n : (r + 1 + rho) mod n;
//                     row shuffle i reads there and writes (i, rho) to (i + rho) mod n.
//   C2R (SoA -> AoS): row shuffle i reads (i, rho) at (i + rho) mod n (the pre-rotation)
//                     and writes it to                i == 0 ? n : (i - 1 + rho) mod n,
//                     where the column pass reads it back.
// Without rotation (c = 1) rho is always 0: the plain rolling scheme.
struct SkinnyRowParams {
    char *A;            // the n x N engine view
    char *tmp;          // location n
    int64_t N;          // row length (the long dimension, count)
    int32_t n, c, b;    // engine rows M = n (fields), c = gcd(n, N), b = N / c
    int64_t ainv;       // a^{-1} mod b, a = n / c
    int32_t i;          // row index
    int32_t T, Tp;      // run length per residue class; shared-memory row pitch (odd)
    int32_t fold;       // 1: the rotation (Eq. 23 / Eq. 36) is folded into the locations
    int32_t reg;        // 1: in-register SIMD transposition kernel (skinny_reg.cu; 4-byte fields)
    unsigned int *gbar; // reg: all n rows in one cooperative launch, grid-barrier counter (zeroed
                        // per launch); null: one launch per row
    FastDiv fd_n, fd_b;
    int64_t batch;      // matrices of the launch (gridDim.y): matrix k at A + k mat_stride,
    int64_t mat_stride, tmp_stride;  // its tmp row at tmp + k tmp_stride (bytes)
};

// Kernel attribute / occupancy caches (api.cu): set the dynamic shared-memory limit (and
// the non-portable cluster flag) once per (kernel, device), and memoise occupancy, so
// that no device query sits between the launches of a call.
cudaError_t ensure_kernel_attrs(const void *kern, size_t smem, bool nonportable_cluster);
int cached_resident_blocks(const void *kern, int threads, size_t smem);  // SMs x blocks per SM

// Group-barrier counters of a column pass: kCtrSlots + 1 words of the CALL's scratch
// (allocated and zeroed in stream order per call, so concurrent calls -- other threads,
// other streams, cudaStreamPerThread -- never share them).  Slots [0, kCtrSlots) are the
// per-tile arrival counters (tile t uses slot t mod kCtrSlots), slot kTicketSlot is the
// dispatch ticket.
constexpr int kCtrSlots = 4096;  // a power of two
constexpr int kTicketSlot = kCtrSlots;
constexpr size_t kCtrBytes = (sizeof(unsigned int) * (kCtrSlots + 1) + 255) & ~size_t(255);
// Copy rows 0..c-2 of every matrix into the wrap buffer (row_shuffle.cu).
cudaError_t launch_copy_wrap(const RowParams &p, int eb, cudaStream_t st);
// Copy the first c-1 rows of every chunk into the boundary rows (chunked fused pass).
cudaError_t launch_copy_bounds(const RowParams &p, int eb, cudaStream_t st);

// Launchers (col_tile.cu / row_shuffle.cu).  They return the CUDA error of the launch.
size_t row_smem_bytes(int64_t N, int eb);
int row_block_threads();
int row_threads(int64_t N, int eb);  // threads per CTA of the one-CTA-per-row-group kernels
cudaError_t launch_row(const RowParams &p, int dir, int eb, cudaStream_t st);
// Fused rotation + row shuffle (p.fuse): shared bytes of one row buffer -- R2C: the row
// (as row_smem_bytes); C2R: c staircase segments of segp bytes + the c-entry pad table.
__host__ __device__ inline size_t row_fused_smem_bytes(const RowParams &p, int eb, int dir) {
    if (dir == ROW_R2C) return (static_cast<size_t>(p.N) * eb + 31) & ~size_t(15);
    return static_cast<size_t>(p.c) * static_cast<size_t>(p.segp) + ((static_cast<size_t>(p.c) * 4 + 15) & ~size_t(15));
}
// Cluster row pass: p.cl_K CTAs per row, each staging cl_seg elements in shared memory,
// gathering through distributed shared memory (row_shuffle.cu).
size_t row_cluster_smem(int32_t seg, int eb);
int row_cluster_active(int K, int32_t seg, int eb, int dir, int mode);  // co-resident clusters (0: none)
cudaError_t launch_row_cluster(const RowParams &p, int dir, int eb, cudaStream_t st);

// Shared memory of a column-pass CTA: nbuf unit buffers (0 or 1: the non-pipelined kernel).
size_t col_smem_bytes(int64_t B, int64_t W, int eb, int nbuf);
int col_max_bufs();
int col_block_threads();
int64_t col_max_band(int64_t W);  // largest band a CTA may be given
cudaError_t launch_col(const ColParams &p, int mode, int eb, cudaStream_t st, size_t smem);
int col_resident_ctas(int mode, int eb, int twb, size_t smem, bool pipe, int threads);

// Skinny column pass (skinny.cu): all n rows x C consecutive columns per CTA, the column
// permutation sigma_j among the n rows applied in shared memory.
struct SkinnyColParams {
    char *A;            // the n x N engine view
    char *tmp;          // the one-row buffer of the rolling scheme
    int64_t N;
    int32_t n, c, b;
    int32_t mode;       // COL_ROT, COL_C2R_SHUF, COL_R2C_SHUF
    int32_t remap;      // +1: output row o stored at o+1 (n-1 in tmp); -1: input row s at s-1 (0 in tmp)
    int32_t fold;       // with remap: + floor(j / b) (mod n) on the rolled side (folded rotation)
    int32_t rot_sign;
    int32_t C;          // columns per CTA (multiple of 32)
    int32_t q[32], qinv[32];  // Eq. 33 / Eq. 34 on the n rows
    FastDiv fd_n, fd_b;
    int64_t batch;      // as SkinnyRowParams
    int64_t mat_stride, tmp_stride;
};
size_t skinny_col_smem(int n, int C, int eb);
cudaError_t launch_skinny_col(const SkinnyColParams &p, int eb, cudaStream_t st);

// Skinny long-row shuffle (skinny.cu): dir ROW_R2C -- dst[d'^{-1}_i(k)] = src[k] driven by
// source windows; dir ROW_C2R -- dst[j] = src[d'^{-1}_i(j)] driven by output windows.
size_t skinny_row_smem(int n, int T, int eb);
cudaError_t launch_skinny_row(const SkinnyRowParams &p, int dir, int eb, cudaStream_t st);
cudaError_t launch_skinny_row_reg(const SkinnyRowParams &p, int dir, cudaStream_t st);

// Record blocks (records.cu, row f3): nblocks = batch * per_mat independent blocks of L
// records of k w-byte words at base + b*mat_stride_bytes + j*blk_stride_bytes; split: L x k
// -> k x L words, merge: k x L -> L x k.  Each block is staged whole: L*k*w bytes of smem,
// or (tmp != null) a slot of global scratch per CTA.
constexpr size_t kRecordSmemMax = 220 * 1024;
constexpr size_t kRecordTmpMax = size_t(1) << 30;  // global-staged blocks: scratch cap
struct RecordParams {
    char *base;
    int64_t nblocks, per_mat, mat_stride_bytes, blk_stride_bytes;
    uint32_t L, k;
    int32_t split;
    FastDiv fd_k, fd_L;  // fd_L: sub-word split of ragged rows
    char *tmp;      // non-null: blocks staged in global scratch, grid slots of L*k*w bytes
    uint32_t grid;  // with tmp: CTAs (= scratch slots)
};
cudaError_t launch_record_blocks(const RecordParams &p, int w, cudaStream_t st);

}  // namespace ipt
