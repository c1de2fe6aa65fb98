// C ABI (include/ipt.h): argument validation, the host planner and pass dispatch.
//
// Planner:
//  * export + layout -> buffer permutation P_{x,y} ("transpose the row-major x-by-y
//    buffer"), Theorems 1-2, reading C18;
//  * engine: C2R(M=x, N=y) if x > y, else R2C(M=y, N=x) -- the paper's heuristic "if
//    m > n, use the C2R algorithm, otherwise use the R2C algorithm" (:959, reading C11):
//    the row length N = min(x, y) is the dimension staged on chip;
//  * constants c = gcd, a, b (:275-277), a^{-1} = mmi(a, b), b^{-1} = mmi(b, a)
//    (:673-685, :719), strength-reduced divisors (§4.4, :745-749);
//  * pass list and launch geometry (row kernel; column-tile width W, band B, group size G).
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>
#include <algorithm>
#include <string>
#include <unordered_map>

#include "ipt.h"
#include "ipt_debug.h"
#include "plan.h"

namespace ipt {
namespace {

std::atomic<uint64_t> g_launches{0};

struct DevInfo {
    int ok = 0;
    int sms = 0, smem_optin = 0, major = 0, minor = 0;
};

DevInfo device_info() {
    static std::mutex mu;
    static DevInfo cache[64];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
        cudaGetLastError();
        return DevInfo{};
    }
    std::lock_guard<std::mutex> lk(mu);
    DevInfo &d = cache[dev];
    if (!d.ok) {
        cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev);
        cudaDeviceGetAttribute(&d.smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        cudaDeviceGetAttribute(&d.major, cudaDevAttrComputeCapabilityMajor, dev);
        cudaDeviceGetAttribute(&d.minor, cudaDevAttrComputeCapabilityMinor, dev);
        d.ok = cudaGetLastError() == cudaSuccess ? 1 : 0;
    }
    return d;
}

int64_t gcd64(int64_t x, int64_t y) {
    while (y) {
        int64_t t = x % y;
        x = y;
        y = t;
    }
    return x;
}

// Modular multiplicative inverse; mmi(x, 1) = 0.
int64_t mmi64(int64_t x, int64_t y) {
    if (y == 1) return 0;
    int64_t r0 = y, r1 = x % y, t0 = 0, t1 = 1;
    while (r1) {
        int64_t q = r0 / r1, t;
        t = r0 - q * r1; r0 = r1; r1 = t;
        t = t0 - q * t1; t0 = t1; t1 = t;
    }
    t0 %= y;
    return t0 < 0 ? t0 + y : t0;
}

int env_int(const char *name, int dflt) {
    const char *v = std::getenv(name);
    return v && *v ? std::atoi(v) : dflt;
}

struct ColPlan {
    ColParams p;
    size_t smem = 0;
    int mode = 0;
};

struct Plan {
    int engine = ENG_NONE;
    int64_t M = 0, N = 0, c = 1, a = 1, b = 1;
    int eb = 4;
    RowParams row{};
    int row_dir = 0;
    ColPlan shuf, rot;
    bool has_rot = false;
    int nlaunch = 0;
    size_t onchip = 0;
    size_t scratch = 0;         // global scratch bytes (skinny: one row of the long dimension)
    size_t side_bytes = 0;      // lagged layouts: side block bytes per matrix (M x (D TWB + pad))
    SkinnyRowParams srow{};     // skinny engine long-row shuffle
    SkinnyColParams scol{}, srot{};  // skinny engine column passes (shuffle, rotation)
    int chunk_force = 0;        // 1: IPT_ROW_CHUNK=1; 2: c = 5..8 (chunks of 8 (c - 1) rows)
    int col_super = 1;          // lagged column pass: super-tile width (col_tile_kernel)
    int sms = 0;
    int skinny_dir = 0;         // ROW_R2C (P_{count,n}, AoS -> SoA) or ROW_C2R (P_{n,count})
    bool skinny_one = false;    // register row shuffles in one cooperative launch
};

int ilog2(int v) {
    int l = 0;
    while ((1 << l) < v) ++l;
    return l;
}

// Column-tile geometry.  Tile width TWB = IPT_TILE_BYTES (128, 256 or 512; default 128 B =
// one cache line).  Band: the rows per CTA that fit the per-CTA shared-memory target
// IPT_COL_SMEM (default 54000 B, four CTAs per SM: the best of the round-1 sweeps over
// 12-100 KiB, profiles/r01_*).  Group size G = ceil(M / B) CTAs per tile; if a group would exceed
// the co-resident CTAs, the band grows (up to the opt-in shared-memory maximum).
ipt_status_t plan_col_v(const DevInfo &dev, const Plan &pl, int mode, ColPlan &cp, bool pipe, int nbuf_min = 2);

// IPT_COL_PIPE (default 0; 1 selects it): the persistent pipelined kernel with IPT_COL_NBUF unit buffers
// per CTA (the shared-memory target is per buffer); tiles whose group would not fit the
// co-resident CTAs that way (very tall matrices, config 5a) take the one-unit kernel.
ipt_status_t plan_col(const DevInfo &dev, const Plan &pl, int mode, ColPlan &cp, bool barrier = false) {
    // Barrier mode (a tile's G units read before any writes: the rotation pass, unlagged
    // shuffles) runs the persistent kernel under a cooperative launch (launch_col), so the
    // group's co-residency is guaranteed by the launch instead of assumed.
    if ((barrier || env_int("IPT_COL_PIPE", 0) != 0) && plan_col_v(dev, pl, mode, cp, true) == IPT_OK) return IPT_OK;
    // very tall tiles: one unit buffer per CTA doubles the co-resident CTAs (G <= grid)
    if (barrier && plan_col_v(dev, pl, mode, cp, true, 1) == IPT_OK) return IPT_OK;
    return plan_col_v(dev, pl, mode, cp, false);
}

ipt_status_t plan_col_v(const DevInfo &dev, const Plan &pl, int mode, ColPlan &cp, bool pipe, int nbuf_min) {
    int twb = env_int("IPT_TILE_BYTES", 128);
    if (twb != 128 && twb != 256 && twb != 512) twb = 128;
    if (pl.M >= (int64_t(1) << 29)) return IPT_ERR_UNSUPPORTED;
    const int nbuf = pipe ? std::min(std::max(nbuf_min == 1 ? 1 : env_int("IPT_COL_NBUF", 2), nbuf_min), col_max_bufs()) : 1;
    const int64_t target = env_int("IPT_COL_SMEM", 54000);
    const int64_t W = twb / pl.eb;
    // Largest band whose buffer fits the target (col_smem_bytes: staged rows + row indices).
    int64_t B = target / (twb + 8);
    while (B > 32 && col_smem_bytes(B, W, pl.eb, 1) > static_cast<size_t>(target)) B -= 8;
    if (B < 32) B = 32;
    if (B > col_max_band(W)) B = col_max_band(W);
    if (B > pl.M) B = pl.M;
    for (;;) {
        const size_t smem = col_smem_bytes(B, W, pl.eb, nbuf);
        if (smem > static_cast<size_t>(dev.smem_optin)) return IPT_ERR_UNSUPPORTED;
        const int64_t G = (pl.M + B - 1) / B;
        const int threads = pipe ? col_block_threads() : static_cast<int>(env_int("IPT_COL_THREADS", 256));
        const int resident = col_resident_ctas(mode, pl.eb, twb, smem, pipe, threads);
        if (resident < 1) return IPT_ERR_UNSUPPORTED;
        if (G > resident) {  // a whole group must be co-resident
            B = (pl.M + resident - 1) / resident;
            if (B > col_max_band(W)) return IPT_ERR_UNSUPPORTED;
            continue;
        }
        ColParams &p = cp.p;
        std::memset(&p, 0, sizeof(p));
        p.M = static_cast<int32_t>(pl.M);
        p.N = static_cast<int32_t>(pl.N);
        p.c = static_cast<int32_t>(pl.c);
        p.a = static_cast<int32_t>(pl.a);
        p.b = static_cast<int32_t>(pl.b);
        p.binv = static_cast<int32_t>(mmi64(pl.b, pl.a));
        p.fd_c = make_fastdiv(static_cast<uint32_t>(pl.c));
        p.fd_a = make_fastdiv(static_cast<uint32_t>(pl.a));
        p.fd_b = make_fastdiv(static_cast<uint32_t>(pl.b));
        p.fd_M = make_fastdiv(static_cast<uint32_t>(pl.M));
        p.W = static_cast<int32_t>(W);
        p.log2W = ilog2(static_cast<int>(W));
        p.ntiles = static_cast<int32_t>((pl.N + W - 1) / W);
        p.G = static_cast<int32_t>(G);
        p.B = static_cast<int32_t>(B);
        p.resident = resident;
        p.pipe = pipe ? 1 : 0;
        p.nbuf = nbuf;
        p.threads = threads;
        p.dbg = env_int("IPT_COL_DEBUG", 0);
        p.rot_sign = 1;
        p.wide_a = pl.a >= 65536 ? 1 : 0;
        cp.smem = smem;
        cp.mode = mode;
        return IPT_OK;
    }
}

// Persistent grid of a column pass over `batch` matrices: as many whole groups as are
// co-resident, never more than there are tiles.
void finish_col(ColParams &p, int64_t batch) {
    if (p.G < 1) return;  // pass not planned (e.g. no rotation when gcd = 1)
    p.fd_G = make_fastdiv(static_cast<uint32_t>(p.G));
    p.fd_nt = make_fastdiv(static_cast<uint32_t>(p.ntiles));
    p.kshM = static_cast<uint32_t>(2 + p.W / p.M) * static_cast<uint32_t>(p.M);
    p.total_tiles = static_cast<int64_t>(p.ntiles) * batch;
    // One-CTA tiles: enough tiles per CTA for ~4 waves of resident CTAs.
    p.tpc = 1;
    if (p.G == 1) {
        const int64_t want = 4 * static_cast<int64_t>(p.resident);
        p.tpc = static_cast<int32_t>(std::max<int64_t>(1, (p.total_tiles + want - 1) / want));
    }
    int64_t ng = p.resident / p.G;
    if (ng > p.total_tiles) ng = p.total_tiles;
    if (ng < 1) ng = 1;
    p.ngroups = static_cast<int32_t>(ng);
}

// Stream-ordered scratch (the skinny engine's tmp row) from a library-owned pool that keeps
// its memory between calls (release threshold = max), one pool per device.
cudaMemPool_t scratch_pool() {
    static std::mutex mu;
    static std::unordered_map<int, cudaMemPool_t> pools;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    auto it = pools.find(dev);
    if (it != pools.end()) return it->second;
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool = nullptr;
    if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    pools[dev] = pool;
    return pool;
}

// Lag of the shuffle pass's tile layout (col_tile.cu "In-place hazard"): D tiles, at most
// ntiles - 1; sets the side-block geometry shared by the column and row passes.
void set_lag(Plan &pl, int64_t D) {
    ColParams &cq = pl.shuf.p;
    RowParams &rp = pl.row;
    D = std::max<int64_t>(1, std::min<int64_t>(D, cq.ntiles - 1));
    const int64_t twb = static_cast<int64_t>(cq.W) * pl.eb;
    cq.lagD = static_cast<int32_t>(D);
    cq.spitch = D * twb + (pl.N * pl.eb) % 16;
    cq.sstride = (pl.M * cq.spitch + 31) & ~int64_t(15);
    rp.shW = static_cast<int32_t>(D * cq.W);
    rp.spitch = cq.spitch;
    rp.sstride = cq.sstride;
    pl.side_bytes = static_cast<size_t>(cq.sstride);
}

// Chunk geometry of the chunked fused pass for a call on `batch` matrices: cK =
// max(R, 8 (c-1), min(IPT_ROW_CHUNK_K (c-1), ceil(M batch / (8 SMs)))) rows -- the boundary
// traffic 2 (c-1) / cK stays <= 25 % of a pass, and about 8 chunks per SM when the call is
// small -- rounded to whole row groups.  Returns whether the batch has >= 2 chunks per SM
// (always true when forced: IPT_ROW_CHUNK=1 uses cK = max(R, IPT_ROW_CHUNK_K (c-1)); for c = 5..8,
// chunk_force 2, the formula's cK when it gives 2 chunks per SM, else max(R, 8 (c-1))).
bool set_chunks(Plan &pl, int64_t batch) {
    RowParams &rp = pl.row;
    // (32: large batches take chunks of up to 32 (c-1) rows -- config 5b row pass +2.5 %; single
    // matrices rarely reach the cap, the sweep is unchanged: profiles/r02_batch_split.txt)
    const int64_t ckmul = env_int("IPT_ROW_CHUNK_K", 32);
    auto apply = [&](int64_t K) {
        K = (K + rp.R - 1) / rp.R * rp.R;
        const int64_t Mr = (pl.M + rp.R - 1) / rp.R * rp.R;
        if (K > Mr) K = Mr;
        rp.cK = static_cast<int32_t>(K);
        rp.nch = static_cast<int32_t>((pl.M + K - 1) / K);
        rp.fd_nch = make_fastdiv(static_cast<uint32_t>(rp.nch));
        return static_cast<int64_t>(rp.nch) * batch >= 2 * static_cast<int64_t>(pl.sms);
    };
    if (pl.chunk_force == 1) {
        apply(std::max<int64_t>(rp.R, ckmul * (pl.c - 1)));
        return true;
    }
    const int64_t per_sm = std::max<int64_t>(1, env_int("IPT_ROW_CHUNK_PER_SM", 8));
    const int64_t par_rows = (pl.M * batch + per_sm * pl.sms - 1) / (per_sm * static_cast<int64_t>(pl.sms));
    if (apply(std::max<int64_t>({static_cast<int64_t>(rp.R), 8 * (pl.c - 1), std::min<int64_t>(ckmul * (pl.c - 1), par_rows)})))
        return true;
    if (pl.chunk_force == 2) {  // c = 5..8 (make_plan): chunks of 8 (c - 1) rows regardless
        apply(std::max<int64_t>(rp.R, 8 * (pl.c - 1)));
        return true;
    }
    return false;
}

// Skinny engine (§6.1): P_{x,y} with min(x, y) = n <= 32 fields
// and a long dimension.  Engine view: n rows x N = max(x, y).  P_{count,n} (AoS -> SoA)
// = R2C(M = n, N = count); P_{n,count} (SoA -> AoS) = C2R(M = n, N = count) (Theorem 2).
ipt_status_t make_skinny_plan(const DevInfo &dev, int64_t x, int64_t y, int eb, Plan &pl) {
    pl.engine = ENG_SKINNY;
    pl.skinny_dir = y < x ? ROW_R2C : ROW_C2R;
    pl.M = y < x ? y : x;
    pl.N = y < x ? x : y;
    if (pl.N >= (int64_t(1) << 31)) return IPT_ERR_UNSUPPORTED;
    pl.c = gcd64(pl.M, pl.N);
    pl.a = pl.M / pl.c;
    pl.b = pl.N / pl.c;
    const int n = static_cast<int>(pl.M);
    // Column passes: all n rows x C columns per CTA (skinny.cu).
    SkinnyColParams &sc = pl.scol;
    std::memset(&sc, 0, sizeof(sc));
    sc.N = pl.N;
    sc.n = n;
    sc.c = static_cast<int32_t>(pl.c);
    sc.b = static_cast<int32_t>(pl.b);
    sc.fd_n = make_fastdiv(static_cast<uint32_t>(n));
    sc.fd_b = make_fastdiv(static_cast<uint32_t>(pl.b));
    // Staging per CTA: >= 40 KB, and >= 3.3 KB contiguous per field row (n x 3328 B, for
    // large n), <= 110 KB (round-2 sweep of IPT_SKINNY_COLBYTES over n = 2..32, gpurun_out r02u).
    const int colbytes = env_int("IPT_SKINNY_COLBYTES", std::min(110000, std::max(40 * 1024, n * 3328)));
    sc.C = std::max(32, static_cast<int>(colbytes / (n * eb)) / 32 * 32);
    for (int i = 0; i < n; ++i) {  // Eq. 33: q(i) = (i N - floor(i/a)) mod n; q^{-1} its inverse
        const int64_t q = ((static_cast<int64_t>(i) * (pl.N % n) - i / pl.a) % n + n) % n;
        sc.q[i] = static_cast<int32_t>(q);
        sc.qinv[q] = i;
    }
    sc.mode = pl.skinny_dir == ROW_R2C ? COL_R2C_SHUF : COL_C2R_SHUF;
    sc.remap = pl.skinny_dir == ROW_R2C ? 1 : -1;
    // c > 1: fold the rotation into the rolling locations (no rotation pass), unless
    // IPT_FUSE_ROT=0.
    const bool fold = pl.c > 1 && env_int("IPT_FUSE_ROT", 1) != 0;
    sc.fold = fold ? 1 : 0;
    pl.onchip = skinny_col_smem(n, sc.C, eb);
    if (pl.onchip > static_cast<size_t>(dev.smem_optin)) return IPT_ERR_UNSUPPORTED;
    if (pl.c > 1 && !fold) {
        pl.srot = sc;
        pl.srot.mode = COL_ROT;
        pl.srot.remap = 0;
        pl.srot.fold = 0;
        pl.srot.rot_sign = pl.skinny_dir == ROW_C2R ? 1 : -1;  // Eq. 23 before / Eq. 36 after
        pl.has_rot = true;
    }
    // Long-row shuffle windows of n * T elements, T a power of two, ~32 KiB of staging.
    SkinnyRowParams &r = pl.srow;
    std::memset(&r, 0, sizeof(r));
    int T = 32;
    while (static_cast<int64_t>(n) * (2 * T) * eb <= 32 * 1024 && 2 * T <= pl.b) T *= 2;
    r.N = pl.N;
    r.n = n;
    r.c = static_cast<int32_t>(pl.c);
    r.b = static_cast<int32_t>(pl.b);
    r.ainv = mmi64(pl.a, pl.b);
    r.T = T;
    r.Tp = T + (32 % n == 0 ? 32 / n : 1);  // residue classes spread over the banks
    r.fd_n = make_fastdiv(static_cast<uint32_t>(n));
    r.fd_b = make_fastdiv(static_cast<uint32_t>(pl.b));
    r.fold = fold ? 1 : 0;
    r.reg = eb == 4 && env_int("IPT_SKINNY_REG", 1) != 0 ? 1 : 0;
    // register row shuffles: all n rows in one cooperative launch (IPT_SKINNY_ONE=0: one per row)
    const bool one = r.reg && env_int("IPT_SKINNY_ONE", 1) != 0;
    const size_t rs = skinny_row_smem(n, r.Tp, eb);
    if (rs > static_cast<size_t>(dev.smem_optin)) return IPT_ERR_UNSUPPORTED;
    if (rs > pl.onchip) pl.onchip = rs;
    pl.scratch = static_cast<size_t>(pl.N) * eb;  // one row of the long dimension
    pl.nlaunch = (one ? 2 : n + 1) + (pl.has_rot ? 1 : 0);
    pl.skinny_one = one;
    return IPT_OK;
}

// P_{x,y} on `batch` matrices.
ipt_status_t make_plan(int64_t x, int64_t y, int eb, Plan &pl) {
    pl = Plan{};
    pl.eb = eb;
    if (x <= 1 || y <= 1) return IPT_OK;  // P_{1,y} and P_{x,1} are the identity
    const DevInfo dev = device_info();
    if (!dev.ok) return IPT_ERR_CUDA;
    if (dev.major != 10 || dev.minor != 0) return IPT_ERR_UNSUPPORTED;  // sm_100 only

    // Skinny shapes (a dimension <= 32, the other long): the specialised engine (§6.1).
    if (std::min(x, y) <= 32 && std::max(x, y) >= env_int("IPT_SKINNY_MIN", 65536))
        return make_skinny_plan(dev, x, y, eb, pl);

    int engine = x > y ? ENG_C2R : ENG_R2C;
    // IPT_ENGINE_RULE=1: the opposite choice (rows = the long dimension, column tiles of
    // the short one) -- the B200 retune study of SURVEY §8 f2.
    if (env_int("IPT_ENGINE_RULE", 0) == 1) engine = x > y ? ENG_R2C : ENG_C2R;
    const char *force = std::getenv("IPT_FORCE_ENGINE");
    if (force && !std::strcmp(force, "c2r")) engine = ENG_C2R;
    if (force && !std::strcmp(force, "r2c")) engine = ENG_R2C;
    pl.engine = engine;
    pl.M = engine == ENG_C2R ? x : y;  // C2R(x, y) = P_{x,y} = R2C(y, x)
    pl.N = engine == ENG_C2R ? y : x;
    if (pl.M >= (int64_t(1) << 31) || pl.N >= (int64_t(1) << 31)) return IPT_ERR_UNSUPPORTED;
    pl.c = gcd64(pl.M, pl.N);
    pl.a = pl.M / pl.c;
    pl.b = pl.N / pl.c;

    // Row pass: one CTA per row while the row fits its shared memory, else (or from
    // IPT_ROW_CLUSTER_MIN row bytes on) a cluster of K CTAs per row.
    size_t rsm = row_smem_bytes(pl.N, eb);
    const int64_t cl_min = env_int("IPT_ROW_CLUSTER_MIN", 0);
    const bool use_cluster = rsm > static_cast<size_t>(dev.smem_optin) || (cl_min > 0 && pl.N * eb >= cl_min);
    RowParams &rp = pl.row;
    std::memset(&rp, 0, sizeof(rp));
    rp.M = static_cast<int32_t>(pl.M);
    rp.N = static_cast<int32_t>(pl.N);
    rp.c = static_cast<int32_t>(pl.c);
    rp.a = static_cast<int32_t>(pl.a);
    rp.b = static_cast<int32_t>(pl.b);
    rp.ainv = static_cast<int32_t>(mmi64(pl.a, pl.b));
    rp.amodb = static_cast<int32_t>(pl.a % pl.b);
    rp.Mn = static_cast<int32_t>(pl.M % pl.N);
    rp.fd_c = make_fastdiv(static_cast<uint32_t>(pl.c));
    rp.fd_b = make_fastdiv(static_cast<uint32_t>(pl.b));
    rp.fd_N = make_fastdiv(static_cast<uint32_t>(pl.N));
    rp.wide = pl.b >= 65536 ? 1 : 0;
    rp.wideN = pl.N >= 65536 ? 1 : 0;
    {
        const int64_t D = 32;  // lane stride of the row walk
        rp.w_dl = static_cast<int32_t>(D % pl.c);
        rp.w_dlb = static_cast<int32_t>((D % pl.c) * pl.b);
        rp.w_dhc = static_cast<int32_t>((static_cast<int64_t>(rp.ainv) * (D / pl.c)) % pl.b);
        rp.w_dh = static_cast<int32_t>(D % pl.b);
        rp.w_dl2 = static_cast<int32_t>(D / pl.b);
        rp.w_ds = static_cast<int32_t>((D / pl.b + ((D % pl.b) * (pl.M % pl.N)) % pl.N) % pl.N);
        rp.c1_step = static_cast<int32_t>(engine == ENG_C2R ? ((D % pl.N) * rp.ainv) % pl.N
                                                            : ((D % pl.N) * (pl.M % pl.N)) % pl.N);
    }
    pl.row_dir = engine == ENG_C2R ? ROW_C2R : ROW_R2C;
    if (use_cluster) {
        // K CTAs per row; the K with the most co-resident CTAs (ties: the smaller K).
        const int forced = env_int("IPT_ROW_CLUSTER_K", 0);
        rp.cl_mode = env_int("IPT_ROW_CLUSTER_MODE", 1);
        int best_ctas = 0;
        for (int K : {2, 4, 8, 16}) {
            if (forced && K != forced) continue;
            const int64_t seg = ((pl.N + K - 1) / K + 31) / 32 * 32;
            const size_t sm = row_cluster_smem(static_cast<int32_t>(seg), eb);
            if (sm > static_cast<size_t>(dev.smem_optin)) continue;
            const int ctas = row_cluster_active(K, static_cast<int32_t>(seg), eb, pl.row_dir, rp.cl_mode) * K;
            if (ctas > best_ctas) {
                best_ctas = ctas;
                rp.cl_K = K;
                rp.cl_seg = static_cast<int32_t>(seg);
                rsm = sm;
            }
        }
        if (best_ctas == 0) return IPT_ERR_UNSUPPORTED;
        rp.fd_seg = make_fastdiv(static_cast<uint32_t>(rp.cl_seg));
        rp.cl_sync = env_int("IPT_ROW_CLUSTER_SYNC", 1);
    }

    // Small gcd: fold the column rotation into the row pass (row_rot_kernel; IPT_FUSE_ROT=0
    // keeps the separate rotation pass).  Global scratch: one flag per row, and for C2R a
    // copy of rows 0..c-2 (the rows the last c-1 staircases wrap onto).
    if (pl.c > 1 && pl.c <= kMaxFuseC && !use_cluster && env_int("IPT_FUSE_ROT", 1) != 0) {
        rp.segp = static_cast<int32_t>(((pl.b * eb + 15) & ~int64_t(15)) + 32);
        rp.fd_cps = make_fastdiv(static_cast<uint32_t>(rp.segp / 16));
        const size_t fsm = row_fused_smem_bytes(rp, eb, pl.row_dir);
        if (fsm <= static_cast<size_t>(dev.smem_optin)) {
            rp.fuse = 1;
            rp.vec = env_int("IPT_ROW_VEC", 1);
            rsm = fsm;
            pl.scratch = static_cast<size_t>(pl.M) * 4 +
                         (engine == ENG_C2R ? static_cast<size_t>(pl.c - 1) * pl.N * eb : 0);
        }
    }

    // Row groups: R consecutive rows per CTA stage while R rows stay within IPT_ROW_STAGE
    // bytes (default 32 KiB), so that short rows still keep enough bytes in flight per SM.
    rp.R = 1;
    if (!use_cluster) {
        const size_t rowbuf = rp.fuse ? row_fused_smem_bytes(rp, eb, pl.row_dir) : row_smem_bytes(pl.N, eb);
        const int nw = row_threads(pl.N, eb) / 32;
        const size_t target = static_cast<size_t>(env_int("IPT_ROW_STAGE", 32768));
        while (rp.R * 2 <= nw && rp.R * 2 * rowbuf <= target) rp.R *= 2;
        rsm = rowbuf * rp.R;
    }
    // Chunked fused pass (row_chunk_kernel; IPT_ROW_CHUNK=0 keeps the flag-based
    // row_rot_kernel): chunks of cK rows, so the boundary copy costs 2 (c-1) / cK of a pass.
    // Used where it measured faster than row_rot_kernel (tools/ab_calls.py, r02j): both row
    // buffers fit (double buffering); cK and the ">= 2 chunks per SM" condition depend on the
    // batch and are settled by set_chunks() (prepare_call).
    const int chunk_env = env_int("IPT_ROW_CHUNK", -1);  // -1 auto, 0 off, 1 force
    const size_t fbuf = rp.fuse ? row_fused_smem_bytes(rp, eb, pl.row_dir) : 0;
    const bool chunk_ok = 2 * rp.R * fbuf <= static_cast<size_t>(env_int("IPT_ROW_DB_MAX", 112 * 1024));
    // c = 5..8: the chunked pass with chunks of 8 (c - 1) rows whatever the chunk count or the
    // row length (single-buffered rows then prefetch the next group into L2): the sweep's
    // c = 5..8 calls 1877 -> 2093 GB/s against the flag-based pass, whose c staircase
    // segments per row dominate; c = 2..4 and c >= 9 keep the rule below (forcing them loses
    // 1-6 %, profiles/r02_ab_chunk_small_c.txt).
    const bool mid_c = pl.c >= 5 && pl.c <= 8;
    if (rp.fuse && (chunk_env == 1 || (chunk_env == -1 && (chunk_ok || mid_c)))) {
        rp.chunk = 1;
        rp.rpitch = ((pl.N * eb + 15) & ~int64_t(15)) + 16;
        pl.chunk_force = chunk_env == 1 ? 1 : chunk_env == -1 && mid_c ? 2 : 0;
        pl.sms = dev.sms;
        set_chunks(pl, 1);
    }
    rp.db_max = env_int("IPT_ROW_DB_MAX", 112 * 1024);
    rp.pipe = env_int("IPT_ROW_PIPE", 1);
    rp.fd_gpm = make_fastdiv(static_cast<uint32_t>((pl.M + rp.R - 1) / rp.R));

    ipt_status_t s = plan_col(dev, pl, engine == ENG_C2R ? COL_C2R_SHUF : COL_R2C_SHUF, pl.shuf);
    if (s != IPT_OK) return s;
    // Lagged tile layouts (col_tile.cu "In-place hazard"; IPT_COL_LAG=0 keeps the per-tile
    // group barrier): the shuffle pass waits only for the previous tile's group, and the
    // row pass reads (R2C) / writes (C2R) the shifted layout with the side tile S of M x TWB
    // bytes per matrix (O(max(m, n)) scratch).  With the cluster row pass only in its L2 mode
    // (row_cluster_l2_kernel reads / writes the lagged layout; the DSMEM mode does not).
    if (env_int("IPT_COL_LAG", 1) != 0 && (!use_cluster || rp.cl_mode == 1) && pl.shuf.p.ntiles >= 2) {
        ColParams &cq = pl.shuf.p;
        cq.lag = engine == ENG_C2R ? LAG_C2R : LAG_R2C;
        // D (IPT_COL_LAGD, default 8 tiles; 0: twice the co-resident CTAs' worth of
        // groups): the round-1 sweep found 4-8 tiles of slack enough to take the wait off
        // the critical path (tools/col_sweep.sh), larger D no better; at most ntiles - 1.
        // Tall tiles (>= 128 bands, e.g. config 5a): units in band-major order within
        // super-tiles of 64 tiles (col_tile_kernel), which needs D >= 64 -- the concurrently
        // running units then share rows instead of each spanning ~1/G of a 140 GB matrix (TLB
        // reach): column pass 2.5 -> 4.4 TB/s on config 5a (gpurun_out r02r); side block
        // M x 64 x 128 B (0.85 % of that matrix).
        const bool tall = cq.G >= 128;
        int64_t D = env_int("IPT_COL_LAGD", tall ? 64 : 8);
        if (D <= 0) D = (2 * static_cast<int64_t>(cq.resident) + cq.G - 1) / cq.G;
        set_lag(pl, D);
        pl.col_super = env_int("IPT_COL_SUPER", tall ? 64 : 1);
        pl.scratch += pl.side_bytes;
    }
    if (pl.shuf.p.lag == LAG_NONE && pl.shuf.p.G > 1 && !pl.shuf.p.pipe) {  // unlagged shuffle: barrier mode
        s = plan_col(dev, pl, engine == ENG_C2R ? COL_C2R_SHUF : COL_R2C_SHUF, pl.shuf, true);
        if (s != IPT_OK) return s;
    }
    pl.onchip = rsm > pl.shuf.smem ? rsm : pl.shuf.smem;
    pl.nlaunch = 2;
    if (pl.c > 1 && !rp.fuse) {
        s = plan_col(dev, pl, COL_ROT, pl.rot, true);
        if (s != IPT_OK) return s;
        pl.rot.p.rot_sign = engine == ENG_C2R ? 1 : -1;
        pl.has_rot = true;
        pl.nlaunch = 3;
        if (pl.rot.smem > pl.onchip) pl.onchip = pl.rot.smem;
    }
    return IPT_OK;
}

// Plan cache: planning queries the device (cluster occupancy) and must not sit between
// the launches of a call.  Keyed by everything make_plan reads.
struct PlanKey {
    int64_t x, y;
    int eb, dev;
    std::string env;
    bool operator==(const PlanKey &o) const {
        return x == o.x && y == o.y && eb == o.eb && dev == o.dev && env == o.env;
    }
};
struct PlanKeyHash {
    size_t operator()(const PlanKey &k) const {
        return std::hash<int64_t>()(k.x * 1000003 + k.y) ^ (std::hash<std::string>()(k.env) << 1) ^
               static_cast<size_t>(k.eb * 131 + k.dev);
    }
};

std::string tunables_key() {
    std::string s;
    for (const char *n : {"IPT_FORCE_ENGINE", "IPT_TILE_BYTES", "IPT_COL_SMEM", "IPT_COL_PIPE", "IPT_COL_NBUF", "IPT_COL_THREADS", "IPT_COL_DEBUG", "IPT_COL_LAG", "IPT_COL_LAGD", "IPT_COL_SUPER", "IPT_COL_TMA", "IPT_COL_BULK", "IPT_COL_PERSIST", "IPT_COL_SIDECAP", "IPT_ROW_STAGE", "IPT_ROW_VEC", "IPT_ROW_DB_MAX", "IPT_ROW_PIPE", "IPT_ROW_CHUNK", "IPT_ROW_CHUNK_K", "IPT_ROW_CHUNK_PER_SM", "IPT_FUSE_ROT", "IPT_ENGINE_RULE",
                          "IPT_SKINNY_MIN", "IPT_SKINNY_REG", "IPT_SKINNY_ONE", "IPT_SKINNY_COLBYTES", "IPT_ROW_CLUSTER_MIN", "IPT_ROW_CLUSTER_K",
                          "IPT_ROW_CLUSTER_SYNC", "IPT_ROW_CLUSTER_MODE"}) {
        const char *v = std::getenv(n);
        s += v ? v : "-";
        s += '|';
    }
    return s;
}

ipt_status_t cached_plan(int64_t x, int64_t y, int eb, Plan &pl) {
    static std::mutex mu;
    static std::unordered_map<PlanKey, Plan, PlanKeyHash> cache;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) {
        cudaGetLastError();
        return IPT_ERR_CUDA;
    }
    PlanKey key{x, y, eb, dev, tunables_key()};
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find(key);
        if (it != cache.end()) {
            pl = it->second;
            return IPT_OK;
        }
    }
    ipt_status_t s = make_plan(x, y, eb, pl);
    if (s == IPT_OK) {
        std::lock_guard<std::mutex> lk(mu);
        if (cache.size() >= 4096) cache.clear();
        cache.emplace(std::move(key), pl);
    }
    return s;
}

ipt_status_t check(cudaError_t e) {
    if (e == cudaSuccess) return IPT_OK;
    cudaGetLastError();
    return IPT_ERR_CUDA;
}

// ---- per-kernel event profiling (ipt_profile_enable / ipt_profile_read) ---------------
enum ProfKind : int { PK_ROW = 0, PK_COL = 1, PK_ROT = 2, PK_SKINNY = 3 };
struct ProfRec {
    int kind = 0;
    double bytes = 0;
    cudaEvent_t start = nullptr, stop = nullptr;
};
std::atomic<int> g_prof_on{0};
std::mutex g_prof_mu;
std::vector<ProfRec> g_prof;

bool profile_begin(ProfRec &r, int kind, double bytes, cudaStream_t st) {
    if (!g_prof_on.load()) return false;
    r.kind = kind;
    r.bytes = bytes;
    if (cudaEventCreate(&r.start) != cudaSuccess || cudaEventCreate(&r.stop) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    cudaEventRecord(r.start, st);
    return true;
}

void profile_end(ProfRec &r, cudaStream_t st) {
    cudaEventRecord(r.stop, st);
    std::lock_guard<std::mutex> lk(g_prof_mu);
    g_prof.push_back(r);
}

// ---- TMA tensor maps of the column pass (pitch % 16 == 0; ColParams::tma) ----------------
using EncodeTiledFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                   const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn encode_tiled() {
    static EncodeTiledFn fn = [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q{};
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess) {
            cudaGetLastError();
            return static_cast<EncodeTiledFn>(nullptr);
        }
        return reinterpret_cast<EncodeTiledFn>(p);
    }();
    return fn;
}

// u32 view of rows of `row_bytes` at `base`, rows `pitch` apart, matrices `mstride` apart
// (rank 3; rank 2 when mstride == 0), grouped in super-rows of g rows (g pitch a multiple of
// 16): dims {((g - 1) pitch + row_bytes) / 4, rows / g(, batch)}, box {32 u32 = 128 B,
// box_rows(, 1)}.
bool make_map(CUtensorMap *m, const char *base, int64_t row_bytes, int64_t rows, int64_t pitch, int64_t batch,
              int64_t mstride, uint32_t box_rows, int g) {
    EncodeTiledFn enc = encode_tiled();
    if (!enc || reinterpret_cast<uintptr_t>(base) % 16 || (g * pitch) % 16 || pitch % 4 || (mstride && mstride % 16))
        return false;
    const cuuint64_t dims[3] = {static_cast<cuuint64_t>(((g - 1) * pitch + row_bytes) / 4),
                                static_cast<cuuint64_t>(rows / g), static_cast<cuuint64_t>(batch)};
    const cuuint64_t strides[2] = {static_cast<cuuint64_t>(g * pitch), static_cast<cuuint64_t>(mstride)};
    const cuuint32_t box[3] = {32, box_rows, 1};
    const cuuint32_t estr[3] = {1, 1, 1};
    const cuuint32_t rank = mstride ? 3 : 2;
    // at least one whole box in each dimension (small matrices keep cp.async)
    if (dims[0] < box[0] || dims[1] < box[1] || dims[0] >= (cuuint64_t(1) << 32) ||
        dims[1] >= (cuuint64_t(1) << 32) || dims[2] >= (cuuint64_t(1) << 32))
        return false;
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT32, rank, const_cast<char *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

int super_rows(int64_t pitch) {  // g = 16 / gcd(pitch, 16) for a pitch that is a multiple of 4
    return pitch % 16 == 0 ? 1 : pitch % 8 == 0 ? 2 : 4;
}

// Enable TMA staging for a shuffle / rotation pass where the layout allows (128-byte tiles,
// 16-byte pitches and bases); otherwise the pass keeps 16-byte cp.async hulls.
// IPT_COL_TMA is a mask of the allowed kinds (default 3): 1 box loads of the matrix, 2 box loads
// of the side block, 4 tile::gather4 for R2C (measured slower than cp.async hulls on the
// sweep: R2C aligned shapes 4688 vs 5005 GB/s, while box loads take C2R from 5148 to 5378;
// tools/ab_calls.py, gpurun_out r02z).
void setup_col_tma(ColParams &p, int mode, int eb) {
    p.tma = 0;
    const int allow = env_int("IPT_COL_TMA", 3);
    if (p.pipe || p.W * eb != 128 || allow == 0) return;
    const int64_t pitch = static_cast<int64_t>(p.N) * eb;
    const bool packed = p.batch == 1 || p.mat_stride_bytes == static_cast<int64_t>(p.M) * pitch;
    if (mode == COL_R2C_SHUF) {
        if ((allow & 4) && packed &&
            make_map(&p.tmap_g, p.base, pitch, static_cast<int64_t>(p.M) * p.batch, pitch, 1, 0, 1, 1))
            p.tma |= 4;
        return;
    }
    if (!(allow & 1)) return;
    // 16-byte pitches only.  (Super-rows of g rows make any pitch a multiple of 16, but their
    // per-phase boxes start at x = p pitch / 4, not 16-byte aligned, and the TMA unit faults on
    // such boxes -- cudaErrorIllegalInstruction on 1024 x 1023 fp32, gpurun_out r02aa; with the
    // box x aligned down and 144-byte hull boxes they are correct but 5 % slower than cp.async
    // hulls, profiles/r02_ab_tma_hull_boxes.txt.)  The kernel's phase logic stays general.
    p.tg_a = super_rows(pitch);
    if (p.tg_a > 1) return;
    p.trows_a = p.M / p.tg_a * p.tg_a;
    // (rank 3 always -- the kernel issues 3-D boxes; one matrix: any 16-byte multiple serves)
    const int64_t ms = p.batch == 1 ? ((static_cast<int64_t>(p.M) * pitch + 15) & ~int64_t(15)) : p.mat_stride_bytes;
    if (make_map(&p.tmap_a, p.base, pitch, p.M, pitch, p.batch, ms, kTmaBoxRows, p.tg_a)) p.tma |= 1;
    if ((allow & 2) && mode == COL_C2R_SHUF && p.lag == LAG_C2R && p.side && (p.tma & 1)) {  // (aligned matrix bases)
        const char *s0 = side_matrix(p.side, p.sstride, 0, p.base);
        p.tg_s = super_rows(p.spitch);
        p.trows_s = p.M / p.tg_s * p.tg_s;
        if (p.tg_s == 1 &&
            make_map(&p.tmap_s, s0, static_cast<int64_t>(p.lagD) * 128, p.M, p.spitch, p.batch, p.sstride,
                     kTmaBoxRows, p.tg_s))
            p.tma |= 2;
    }
}

// ---- per-call global scratch (Theorem 6: O(max(m, n)) per worker) -------------------
// One stream-ordered allocation per call, laid out as
//   [ counters: shuffle pass | rotation pass ][ row flags + ticket ]   <- zeroed (one memset)
//   [ wrap rows ][ side blocks ]  or, for the skinny engine, [ tmp row ]
// Nothing is shared between calls, so concurrent calls (other host threads, other
// streams, cudaStreamPerThread) cannot see each other's counters.
struct CallScratch {
    size_t ctr_shuf = 0, ctr_rot = 0;  // column-pass counter blocks (kCtrBytes each)
    size_t flags = 0;                  // fused rotation: M*batch row flags + the ticket
    size_t zero_bytes = 0;             // [0, zero_bytes) is zeroed before the first pass
    size_t gbar = 0;                   // skinny engine: grid-barrier counter of the one-launch row pass
    size_t wrap = 0, wstride = 0;      // fused rotation: per-matrix copy of rows 0..c-2
    size_t bnd = 0;                    // chunked fused pass: boundary rows
    size_t side = 0;                   // lagged layouts: side blocks
    size_t total = 0;
};

size_t al256(size_t x) { return (x + 255) & ~size_t(255); }

// Skinny batches: matrices per launch, each needing one tmp row of N eb bytes -- the tmp rows of
// a launch stay within 256 MiB (at least one matrix), at most 65535 (gridDim.y).
int64_t skinny_sub(const Plan &pl, int64_t batch) {
    const int64_t row = std::max<int64_t>(1, pl.N * pl.eb);
    return std::max<int64_t>(1, std::min<int64_t>({batch, (int64_t(256) << 20) / row, 65535}));
}

// Final plan of a call on `batch` matrices (batches cap the lag) and its scratch layout.
// Pure host arithmetic: nothing is enqueued.
void prepare_call(Plan &pl, int64_t batch, CallScratch &cs) {
    cs = CallScratch{};
    if (pl.engine == ENG_NONE || batch == 0) return;
    if (pl.engine == ENG_SKINNY) {
        cs.total = al256(pl.scratch * static_cast<size_t>(skinny_sub(pl, batch)));
        if (pl.skinny_one) {  // grid-barrier counter of the one-launch row shuffles (zeroed per launch)
            cs.gbar = cs.total;
            cs.total += 256;
        }
        return;
    }
    const double full = 2.0 * static_cast<double>(pl.M) * static_cast<double>(pl.N) * pl.eb * static_cast<double>(batch);
    if (pl.side_bytes && batch > 1) {
        // Batches: keep the side blocks within max(256 MiB, 1/8 of the data) -- a smaller D
        // beyond that.  (1/32 forced D = 2 on config 5b's 512-matrix chunks and the column pass
        // waited on its lag: 4378 -> 4878 GB/s, call 2389 -> 2531 GB/s with 1/8;
        // profiles/r02_batch_sidecap.txt.  D = 8 tiles of 128 B is 256 / N of the data.)
        const double cap = std::max(256.0 * (1 << 20), full / 2.0 / static_cast<double>(env_int("IPT_COL_SIDECAP", 8)));
        const double per_tile = static_cast<double>(pl.M) * pl.shuf.p.W * pl.eb * static_cast<double>(batch);
        const int64_t dmax = static_cast<int64_t>(cap / per_tile);
        if (dmax < pl.shuf.p.lagD) set_lag(pl, dmax);
    }
    if (pl.row.fuse && pl.row.chunk && !set_chunks(pl, batch))
        pl.row.chunk = 0;  // too few chunks for the GPU: the flag-based fused pass
    size_t o = 0;
    cs.ctr_shuf = o;
    o += kCtrBytes;
    if (pl.has_rot) {
        cs.ctr_rot = o;
        o += kCtrBytes;
    }
    const bool flagged = pl.row.fuse && !pl.row.chunk;  // row_rot_kernel / pipelined fused pass
    if (flagged) {
        cs.flags = o;
        o += al256((static_cast<size_t>(pl.M) * static_cast<size_t>(batch) + 1) * 4);
    }
    cs.zero_bytes = o;
    if (flagged) {
        cs.wrap = o;
        cs.wstride = al256(static_cast<size_t>(pl.c - 1) * pl.N * pl.eb + 16);
        o += cs.wstride * static_cast<size_t>(batch);
    }
    if (pl.row.fuse && pl.row.chunk) {
        cs.bnd = o;
        o += al256(static_cast<size_t>(pl.row.nch) * static_cast<size_t>(batch) * static_cast<size_t>(pl.c - 1) *
                   static_cast<size_t>(pl.row.rpitch));
    }
    if (pl.side_bytes) {
        cs.side = o;
        o += pl.side_bytes * static_cast<size_t>(batch);
    }
    cs.total = o;
}

ipt_status_t pool_alloc(char **p, size_t bytes, cudaStream_t st) {
    *p = nullptr;
    if (!bytes) return IPT_OK;
    cudaMemPool_t pool = scratch_pool();
    if (!pool || cudaMallocFromPoolAsync(reinterpret_cast<void **>(p), bytes, pool, st) != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return IPT_ERR_OUT_OF_MEMORY;
    }
    return IPT_OK;
}

// Enqueue the passes of a prepared call.  `scratch` holds cs.total bytes (stream-ordered,
// owned by the caller of this function).
ipt_status_t launch_call(const Plan &pl0, const CallScratch &cs, char *base, int64_t batch, int64_t stride_bytes,
                         cudaStream_t st, char *scratch) {
    if (pl0.engine == ENG_NONE || batch == 0) return IPT_OK;
    Plan pl = pl0;
    // Row groups are numbered in 32 bits (row_shuffle.cu row_group, the fused pass's ticket).
    if (pl.engine != ENG_SKINNY && (pl.M + pl.row.R - 1) / pl.row.R * batch >= (int64_t(1) << 32) - 1)
        return IPT_ERR_UNSUPPORTED;
    pl.row.base = base;
    pl.row.batch = batch;
    pl.row.mat_stride_bytes = stride_bytes;
    for (ColPlan *cp : {&pl.shuf, &pl.rot}) {
        cp->p.base = base;
        cp->p.batch = batch;
        cp->p.mat_stride_bytes = stride_bytes;
        finish_col(cp->p, batch);
    }
    // IPT_DEBUG_PASSES=k (tests only): stop after the first k passes, so that each pass
    // can be compared with the oracle's snapshot of the same step.
    int budget = env_int("IPT_DEBUG_PASSES", 1 << 30);
    const double full = 2.0 * static_cast<double>(pl.M) * static_cast<double>(pl.N) * pl.eb * static_cast<double>(batch);
    auto run = [&](int kind, double bytes, auto &&launch) -> ipt_status_t {
        if (budget-- <= 0) return IPT_OK;
        ProfRec rec;
        const bool prof = profile_begin(rec, kind, bytes, st);
        ipt_status_t s = check(launch());
        if (prof) profile_end(rec, st);
        if (s == IPT_OK) g_launches++;
        return s;
    };
    ipt_status_t s;
    if (pl.engine == ENG_SKINNY) {
        // Rolling rows (§6.1; DESIGN.md §"Skinny"): engine view n rows x N, one
        // tmp row of N elements.  R2C: column pass writing row r to location r+1 (row n-1 to
        // tmp); row i then reads location i+1 (tmp for n-1) and writes location i.  C2R:
        // row i reads location i, writes location i-1 (tmp for 0); the column pass reads the
        // shifted rows back.  A destination row is never its own source row.  With c > 1 the
        // rotation is folded in: block rho = floor(j/b) of every rolled location is shifted
        // by another rho rows (plan.h, SkinnyRowParams).
        // Batches: every pass is one launch for a sub-batch of up to skinny_sub(...) matrices
        // (gridDim.y = matrix, each with its own tmp row in the call's scratch).
        const int n = static_cast<int>(pl.M);
        const int64_t sub = skinny_sub(pl, batch);
        const double rowb = 2.0 * static_cast<double>(pl.N) * pl.eb;
        char *tmp = scratch;
        s = IPT_OK;
        for (int64_t mat = 0; mat < batch; mat += sub) {
            const int64_t nb = std::min(sub, batch - mat);
            char *A = base + mat * stride_bytes;
            SkinnyColParams shuf = pl.scol, rotp = pl.srot;
            shuf.A = rotp.A = A;
            shuf.tmp = rotp.tmp = tmp;
            shuf.batch = rotp.batch = nb;
            shuf.mat_stride = rotp.mat_stride = stride_bytes;
            shuf.tmp_stride = rotp.tmp_stride = pl.N * pl.eb;
            auto rot_l = [&] { return launch_skinny_col(rotp, pl.eb, st); };
            auto shuf_l = [&] { return launch_skinny_col(shuf, pl.eb, st); };
            const bool one = pl.skinny_one;  // all rows in one cooperative launch
            unsigned int *gbar = one ? reinterpret_cast<unsigned int *>(scratch + cs.gbar) : nullptr;
            auto row_l = [&](int i) {
                SkinnyRowParams rp = pl.srow;
                rp.i = i;
                rp.gbar = gbar;
                rp.A = A;
                rp.tmp = tmp;
                rp.batch = nb;
                rp.mat_stride = stride_bytes;
                rp.tmp_stride = pl.N * pl.eb;
                return [rp, &pl, st] { return launch_skinny_row(rp, pl.skinny_dir, pl.eb, st); };
            };
            auto rows = [&]() -> ipt_status_t {
                if (!one) {
                    ipt_status_t r = IPT_OK;
                    for (int i = 0; i < n && r == IPT_OK; ++i) r = run(PK_SKINNY, rowb, row_l(i));
                    return r;
                }
                ipt_status_t r = check(cudaMemsetAsync(gbar, 0, sizeof(unsigned int), st));
                return r == IPT_OK ? run(PK_SKINNY, rowb * n, row_l(0)) : r;
            };
            if (pl.skinny_dir == ROW_R2C) {
                if ((s = run(PK_COL, rowb * n, shuf_l)) != IPT_OK) break;
                s = rows();
                if (s == IPT_OK && pl.has_rot) s = run(PK_ROT, rowb * n, rot_l);
            } else {
                if (pl.has_rot && (s = run(PK_ROT, rowb * n, rot_l)) != IPT_OK) break;
                s = rows();
                if (s == IPT_OK) s = run(PK_COL, rowb * n, shuf_l);
            }
            if (s != IPT_OK) break;
        }
        return s;
    }
    // Column-pass counters, fused-rotation flags + ticket: zeroed in stream order -- by the row
    // kernel when a pipelined / chunked C2R row pass is the call's first kernel (the counters
    // are then its only zeroed state), else by a memset.
    const bool row_zeroes = pl.engine == ENG_C2R && !pl.has_rot && pl.row.pipe && !pl.row.cl_K &&
                            (!pl.row.fuse || pl.row.chunk) && env_int("IPT_DEBUG_PASSES", 1 << 30) >= (1 << 30);
    if (row_zeroes) {
        pl.row.zero = reinterpret_cast<unsigned int *>(scratch + cs.ctr_shuf);
        pl.row.zero_words = static_cast<int32_t>(cs.zero_bytes / 4);
    } else if (cs.zero_bytes && (s = check(cudaMemsetAsync(scratch, 0, cs.zero_bytes, st))) != IPT_OK) {
        return s;
    }
    pl.shuf.p.ctr = reinterpret_cast<unsigned int *>(scratch + cs.ctr_shuf);
    pl.rot.p.ctr = reinterpret_cast<unsigned int *>(scratch + cs.ctr_rot);
    pl.shuf.p.ticket = pl.rot.p.ticket = env_int("IPT_COL_TICKET", 1) != 0 ? 1 : 0;
    // super-tiles (lagged shuffle pass only; S <= D keeps every wait on a smaller ticket, and
    // the band-major order needs the ticket)
    pl.shuf.p.super = 1;
    if (pl.shuf.p.lag != LAG_NONE && pl.shuf.p.ticket && pl.shuf.p.G > 1)
        pl.shuf.p.super = std::max(1, std::min<int>(pl.col_super, pl.shuf.p.lagD));
    if (pl.row.fuse && !pl.row.chunk) {
        pl.row.flags = reinterpret_cast<unsigned int *>(scratch + cs.flags);
        pl.row.ticket = pl.row.flags + pl.M * batch;
        pl.row.wrap = scratch + cs.wrap;
        pl.row.wstride = static_cast<int64_t>(cs.wstride);
    }
    if (pl.row.fuse && pl.row.chunk) {
        if (static_cast<int64_t>(pl.row.nch) * batch >= (int64_t(1) << 32)) return IPT_ERR_UNSUPPORTED;
        pl.row.bnd = scratch + cs.bnd;
    }
    pl.row.side = pl.shuf.p.side = pl.side_bytes ? scratch + cs.side : nullptr;
    setup_col_tma(pl.shuf.p, pl.engine == ENG_C2R ? COL_C2R_SHUF : COL_R2C_SHUF, pl.eb);
    pl.shuf.p.bulk = !pl.shuf.p.pipe && pl.shuf.p.W * pl.eb == 128 && env_int("IPT_COL_BULK", 0) != 0 ? 1 : 0;
    pl.shuf.p.persist = pl.shuf.p.lag != LAG_NONE && pl.shuf.p.G > 1 && pl.shuf.p.ticket && !pl.shuf.p.pipe &&
                        env_int("IPT_COL_PERSIST", 1) != 0 ? 1 : 0;  // sweep: calls +3.1 %, R2C shuffles +13 % (r02ae)
    if (pl.has_rot) setup_col_tma(pl.rot.p, COL_ROT, pl.eb);
    const int64_t pitch = pl.N * pl.eb;
    const int passes = budget;
    // The rotation moves only the columns with a non-zero amount: (c - 1) / c of them.
    const double rot_bytes = full * static_cast<double>(pl.c - 1) / static_cast<double>(pl.c);
    auto rot = [&] { return launch_col(pl.rot.p, COL_ROT, pl.eb, st, pl.rot.smem); };
    auto row = [&] {
        if (pl.row.fuse) {  // chunk boundary rows / rows 0..c-2 of every matrix copied first
            cudaError_t e = pl.row.chunk ? launch_copy_bounds(pl.row, pl.eb, st) : launch_copy_wrap(pl.row, pl.eb, st);
            if (e != cudaSuccess) return e;
            g_launches++;
        }
        return pl.row.cl_K ? launch_row_cluster(pl.row, pl.row_dir, pl.eb, st) : launch_row(pl.row, pl.row_dir, pl.eb, st);
    };
    if (pl.engine == ENG_C2R) {
        auto shuf = [&] { return launch_col(pl.shuf.p, COL_C2R_SHUF, pl.eb, st, pl.shuf.smem); };
        if (pl.has_rot && (s = run(PK_ROT, rot_bytes, rot)) != IPT_OK) return s;  // Eq. 23
        if ((s = run(PK_ROW, full, row)) != IPT_OK) return s;                     // Eq. 31
        if ((s = run(PK_COL, full, shuf)) != IPT_OK) return s;                    // Eq. 26
    } else {
        auto shuf = [&] { return launch_col(pl.shuf.p, COL_R2C_SHUF, pl.eb, st, pl.shuf.smem); };
        if ((s = run(PK_COL, full, shuf)) != IPT_OK) return s;                    // Eqs. 34-35
        if ((s = run(PK_ROW, full, row)) != IPT_OK) return s;                     // Eq. 24
        if (pl.has_rot && (s = run(PK_ROT, rot_bytes, rot)) != IPT_OK) return s;  // Eq. 36
    }
    // IPT_DEBUG_PASSES stopping between the row and column passes of a lagged plan: put the
    // logical layout back (side tile -> columns [0, W), A columns [0, N - W) -> [W, N)) so
    // the snapshot compares with the oracle's.  Tests only (small matrices).
    if (pl.side_bytes && passes < (1 << 30)) {
        const int before_second = pl.engine == ENG_C2R ? (pl.has_rot ? 2 : 1) : 1;  // passes up to the lagged state
        if (passes == before_second) {
            const size_t W = static_cast<size_t>(pl.row.shW), sp = static_cast<size_t>(pl.row.spitch);
            char *tmp = nullptr;
            if (cudaMallocAsync(reinterpret_cast<void **>(&tmp), static_cast<size_t>(pitch) * pl.M, st) != cudaSuccess)
                return IPT_ERR_OUT_OF_MEMORY;
            for (int64_t k = 0; k < batch && s == IPT_OK; ++k) {
                char *A = base + k * stride_bytes;
                s = check(cudaMemcpy2DAsync(tmp + W * pl.eb, pitch, A, pitch, pitch - W * pl.eb, pl.M,
                                            cudaMemcpyDeviceToDevice, st));
                if (s == IPT_OK)
                    s = check(cudaMemcpy2DAsync(tmp, pitch, side_matrix(pl.row.side, pl.row.sstride, k, A), sp,
                                                W * pl.eb, pl.M, cudaMemcpyDeviceToDevice, st));
                if (s == IPT_OK)
                    s = check(cudaMemcpyAsync(A, tmp, static_cast<size_t>(pitch) * pl.M, cudaMemcpyDeviceToDevice, st));
            }
            cudaFreeAsync(tmp, st);
            return s;
        }
    }
    return IPT_OK;
}

// A resolved engine call: plan, scratch layout; run = allocate + launch + free.
struct Call {
    Plan pl;
    CallScratch cs;
    int64_t batch = 0;
};

ipt_status_t resolve(int64_t x, int64_t y, int eb, int64_t batch, Call &c) {
    c = Call{};
    c.batch = batch;
    if (x <= 1 || y <= 1 || batch == 0) return IPT_OK;  // identity: engine NONE
    ipt_status_t s = cached_plan(x, y, eb, c.pl);
    if (s != IPT_OK) return s;
    prepare_call(c.pl, batch, c.cs);
    return IPT_OK;
}

ipt_status_t launch_resolved(const Call &c, char *base, int64_t stride_bytes, cudaStream_t st, char *scratch) {
    return launch_call(c.pl, c.cs, base, c.batch, stride_bytes, st, scratch);
}

ipt_status_t run_resolved(const Call &c, char *base, int64_t stride_bytes, cudaStream_t st) {
    char *scratch = nullptr;
    ipt_status_t s = pool_alloc(&scratch, c.cs.total, st);
    if (s != IPT_OK) return s;
    s = launch_resolved(c, base, stride_bytes, st, scratch);
    if (scratch) cudaFreeAsync(scratch, st);
    return s;
}

bool valid_eb(int eb) { return eb == 4 || eb == 8 || eb == 16; }

// Shared argument checks of every entry point: sizes, strides, overflow, pointer.  Returns
// IPT_OK with `done` set when there is nothing to do (empty / identity).
ipt_status_t check_args(void *ptr, int64_t batch, int64_t &stride, int64_t x, int64_t y, int64_t eb, int64_t align,
                        bool &done) {
    done = false;
    if (x < 0 || y < 0 || batch < 0) return IPT_ERR_INVALID_ARGUMENT;
    if (x != 0 && y > INT64_MAX / x) return IPT_ERR_INVALID_ARGUMENT;
    const int64_t elems = x * y;
    if (stride < 0) stride = elems;
    if (stride < elems) return IPT_ERR_INVALID_ARGUMENT;
    if (stride != 0 && batch > INT64_MAX / stride) return IPT_ERR_INVALID_ARGUMENT;
    if (elems != 0 && batch * stride > INT64_MAX / eb) return IPT_ERR_INVALID_ARGUMENT;
    if (elems == 0 || batch == 0) {
        done = true;
        return IPT_OK;
    }
    if (ptr == nullptr || reinterpret_cast<uintptr_t>(ptr) % static_cast<uintptr_t>(align) != 0)
        return IPT_ERR_INVALID_ARGUMENT;
    if (x <= 1 || y <= 1) done = true;  // P_{1,y} and P_{x,1} are the identity
    return IPT_OK;
}

// Validate and run P_{x,y} on `batch` matrices of x*y elements, `stride` elements apart.
// stride < 0 means "packed" (stride = x*y), used by the single-matrix entry points.
ipt_status_t run_perm(void *ptr, int64_t batch, int64_t stride, int64_t x, int64_t y, int eb, void *stream) {
    if (!valid_eb(eb)) return IPT_ERR_INVALID_ARGUMENT;
    bool done = false;
    ipt_status_t s = check_args(ptr, batch, stride, x, y, eb, eb, done);
    if (s != IPT_OK || done) return s;
    Call c;
    if ((s = resolve(x, y, eb, batch, c)) != IPT_OK) return s;
    return run_resolved(c, static_cast<char *>(ptr), stride * eb, static_cast<cudaStream_t>(stream));
}

// Multi-word elements (the paper's passes move opaque words whatever their
// size, :1037, :1085).  An element of eb = k*w bytes (w = 16, 8 or 4: the largest that
// divides both eb and the base address) is moved by two word-level permutations of the
// engine: P_{x,y} on k-word elements = P_{x,y*k} on words (output row j*k + v holds word v
// of column j), then P_{k,x} on each of the y k-by-x blocks (block j becomes x rows of k
// words, i.e. row j of the y-by-x result).  Buffer traffic: twice the one-step engine.
constexpr int kMaxElemBytes = 4096;

// Staging of the record-block pass for blocks of blk_bytes: slots = 0 in shared memory;
// slots > 0 CTAs each with a global scratch slot (at least one per SM, up to 4, while the
// slots fit ~96 MB and stay L2-resident, never more than the blocks); slots = -1 when even
// one slot per SM would exceed kRecordTmpMax (then both steps run on the engine).
ipt_status_t record_slots(int64_t blk_bytes, int64_t nblocks, int64_t &slots) {
    slots = 0;
    if (env_int("IPT_RECORD_ENGINE", 0)) {  // tests: force both steps onto the engine
        slots = -1;
        return IPT_OK;
    }
    if (blk_bytes <= static_cast<int64_t>(kRecordSmemMax)) return IPT_OK;
    int dev = 0, sms = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
        cudaGetLastError();
        return IPT_ERR_CUDA;
    }
    slots = std::min<int64_t>(nblocks, std::max<int64_t>(sms, std::min<int64_t>(4 * sms, (96ll << 20) / blk_bytes)));
    if (slots * blk_bytes > static_cast<int64_t>(kRecordTmpMax)) slots = -1;
    return IPT_OK;
}
bool valid_multiword_eb(int eb) { return eb > 0 && eb % 4 == 0 && eb <= kMaxElemBytes && !valid_eb(eb); }

int word_bytes_of(int eb, uintptr_t addr) {
    for (int w : {16, 8}) if (eb % w == 0 && addr % w == 0) return w;
    return 4;
}

// A composed call (records, sub-word elements): up to two engine steps and one record-block
// pass, all resolved (plans, scratch sizes, UNSUPPORTED checks) before anything is
// enqueued, with ONE scratch allocation for all of them -- so IPT_ERR_UNSUPPORTED and
// IPT_ERR_OUT_OF_MEMORY leave the buffer untouched, as ipt.h promises.
struct Composed {
    Call e1, e2;                // engine steps (e2 only for the all-engine fallback)
    int64_t e1_stride = 0, e2_stride = 0;  // matrix strides of the engine steps, bytes
    bool blocks = false;        // a record-block pass
    bool blocks_first = false;  // the block pass runs before e1 (merge / split orientation)
    RecordParams rp{};
    int rec_w = 4;              // launch_record_blocks word argument
    size_t rec_tmp = 0;         // global slots of the block pass
    int64_t e2_loops = 0;       // e2 per matrix (strided batch): > 0 loops this many times
    int64_t e2_mat_stride = 0;  // bytes between those matrices
};

ipt_status_t run_composed(const Composed &C, char *base, cudaStream_t st) {
    const size_t s1 = C.e1.cs.total, s2 = C.e2.cs.total;
    const size_t o_rec = al256(std::max(s1, s2));
    char *scratch = nullptr;
    ipt_status_t s = pool_alloc(&scratch, o_rec + C.rec_tmp, st);
    if (s != IPT_OK) return s;
    auto blocks = [&]() -> ipt_status_t {
        RecordParams rp = C.rp;
        rp.tmp = C.rec_tmp ? scratch + o_rec : nullptr;
        ipt_status_t r = check(launch_record_blocks(rp, C.rec_w, st));
        if (r == IPT_OK) g_launches++;
        return r;
    };
    if (C.blocks && C.blocks_first) s = blocks();
    if (s == IPT_OK) s = launch_resolved(C.e1, base, C.e1_stride, st, scratch);
    if (s == IPT_OK && C.blocks && !C.blocks_first) s = blocks();
    if (s == IPT_OK && C.e2.batch) {
        if (C.e2_loops == 0) {
            s = launch_resolved(C.e2, base, C.e2_stride, st, scratch);
        } else {
            for (int64_t b = 0; b < C.e2_loops && s == IPT_OK; ++b)
                s = launch_resolved(C.e2, base + b * C.e2_mat_stride, C.e2_stride, st, scratch);
        }
    }
    if (scratch) cudaFreeAsync(scratch, st);
    return s;
}

// Sub-word elements (1 or 2 bytes): g = 4 / eb elements share one 4-byte
// engine word.  y % g == 0: P_{x,y/g} on words (row j' holds x g-tuples of row elements
// g*j' .. g*j'+g-1), then split each row's x-by-g tuples into g rows of x elements.
// Otherwise x % g == 0: merge each group of g rows (g-by-y elements -> y g-tuples), then
// P_{x/g,y} on words (word (j, i') holds elements (g*i'+v, j), i.e. row j of the result).
// Both x and y indivisible by g is unsupported, as are blocks beyond the record pass's
// scratch budget and batch strides that are not a whole number of words.
bool valid_subword_eb(int eb) { return eb == 1 || eb == 2; }

ipt_status_t resolve_subword(int64_t batch, int64_t stride, int64_t x, int64_t y, int eb, Composed &C) {
    const int64_t g = 4 / eb;
    // Of the feasible orientations, the one with the shorter blocks (L = x for split, y for merge).
    const bool split = y % g == 0 && (x % g != 0 || x <= y);
    if ((!split && x % g != 0) || (batch > 1 && stride % g != 0)) return IPT_ERR_UNSUPPORTED;
    const int64_t L = split ? x : y, per_mat = split ? y / g : x / g, nblocks = batch * per_mat;
    int64_t slots = 0;
    if (record_slots(L * 4, nblocks, slots) != IPT_OK) return IPT_ERR_CUDA;
    if (slots < 0 || L * g >= (int64_t(1) << 32)) return IPT_ERR_UNSUPPORTED;
    RecordParams &rp = C.rp;
    rp = RecordParams{};
    rp.per_mat = per_mat;
    rp.nblocks = nblocks;
    rp.mat_stride_bytes = stride * eb;
    rp.blk_stride_bytes = L * 4;
    rp.L = static_cast<uint32_t>(L);
    rp.k = static_cast<uint32_t>(g);
    rp.split = split;
    rp.fd_k = make_fastdiv(static_cast<uint32_t>(g));
    rp.fd_L = make_fastdiv(static_cast<uint32_t>(L));
    rp.grid = static_cast<uint32_t>(slots);
    C.blocks = true;
    C.blocks_first = !split;
    C.rec_w = eb;
    C.rec_tmp = static_cast<size_t>(slots * L * 4);
    C.e1_stride = stride / g * 4;
    return split ? resolve(x, y / g, 4, batch, C.e1) : resolve(x / g, y, 4, batch, C.e1);
}

ipt_status_t resolve_multiword(int64_t batch, int64_t stride, int64_t x, int64_t y, int eb, uintptr_t addr,
                               Composed &C) {
    const int w = word_bytes_of(eb, addr);
    const int64_t k = eb / w;
    const int64_t L = std::min(x, y);
    const int64_t per_mat = std::max(x, y), nblocks = batch * per_mat;
    int64_t slots = 0;
    if (record_slots(L * eb, nblocks, slots) != IPT_OK) return IPT_ERR_CUDA;
    C.e1_stride = stride * eb;  // = stride * k words of w bytes
    if (slots >= 0 && nblocks < (int64_t(1) << 40)) {
        // The block step on the shorter side, staged in shared memory (records.cu):
        //   x <= y: P_{x,y*k} on words, then merge each k-by-x block into x records;
        //   x >  y: split each row of y records into k-by-y words, then P_{x*k,y} on words
        //           (row i*k + v holds word v of row i, so P_{x*k,y} leaves record (i,j)
        //           at row j, words i*k .. i*k+k-1).
        RecordParams &rp = C.rp;
        rp = RecordParams{};
        rp.per_mat = per_mat;
        rp.nblocks = nblocks;
        rp.mat_stride_bytes = stride * eb;
        rp.blk_stride_bytes = L * eb;
        rp.L = static_cast<uint32_t>(L);
        rp.k = static_cast<uint32_t>(k);
        rp.split = x > y;
        rp.fd_k = make_fastdiv(static_cast<uint32_t>(k));
        rp.grid = static_cast<uint32_t>(slots);
        C.blocks = true;
        C.blocks_first = x > y;
        C.rec_w = w;
        C.rec_tmp = static_cast<size_t>(slots * L * eb);
        return x <= y ? resolve(x, y * k, w, batch, C.e1) : resolve(x * k, y, w, batch, C.e1);
    }
    // Blocks too long for one CTA: both steps on the engine, P_{x, y k} then P_{k, x} on
    // every k-by-x block.
    ipt_status_t s = resolve(x, y * k, w, batch, C.e1);
    if (s != IPT_OK) return s;
    if (batch == 1 || stride == x * y) {  // every k-by-x block of every matrix is k*x words apart
        C.e2_stride = k * x * w;
        return resolve(k, x, w, batch * y, C.e2);
    }
    C.e2_stride = k * x * w;
    C.e2_loops = batch;
    C.e2_mat_stride = stride * eb;
    return resolve(k, x, w, y, C.e2);
}

ipt_status_t run_perm_any(void *ptr, int64_t batch, int64_t stride, int64_t x, int64_t y, int eb, void *stream) {
    if (valid_eb(eb)) return run_perm(ptr, batch, stride, x, y, eb, stream);
    if (!valid_subword_eb(eb) && !valid_multiword_eb(eb)) return IPT_ERR_INVALID_ARGUMENT;
    bool done = false;
    ipt_status_t s = check_args(ptr, batch, stride, x, y, eb, 4, done);
    if (s != IPT_OK || done) return s;
    Composed C;
    s = valid_subword_eb(eb) ? resolve_subword(batch, stride, x, y, eb, C)
                             : resolve_multiword(batch, stride, x, y, eb, reinterpret_cast<uintptr_t>(ptr), C);
    if (s != IPT_OK) return s;
    C.rp.base = static_cast<char *>(ptr);
    return run_composed(C, static_cast<char *>(ptr), static_cast<cudaStream_t>(stream));
}

// Plan description of a single-word call: the plan, with pl.scratch = the bytes the call
// allocates (CallScratch of one matrix).
ipt_status_t engine_plan(int64_t x, int64_t y, int eb, Plan &pl) {
    ipt_status_t s = make_plan(x, y, eb, pl);
    if (s != IPT_OK) return s;
    CallScratch cs;
    prepare_call(pl, 1, cs);
    pl.scratch = cs.total;
    return IPT_OK;
}

// Plan description of a record / sub-word call P_{x,y} (16-byte-aligned base assumed, one
// matrix): `pl` is the plan of its (first) word-level engine step, widened by the other
// steps' scratch and staging; `extra` counts the other steps' launches.  Same resolution
// as the run (resolve_subword / resolve_multiword), so UNSUPPORTED agrees with execution.
ipt_status_t record_plan(int64_t x, int64_t y, int eb, Plan &pl, int64_t &extra) {
    if (x < 0 || y < 0) return IPT_ERR_INVALID_ARGUMENT;
    if (x != 0 && y > INT64_MAX / x) return IPT_ERR_INVALID_ARGUMENT;
    pl = Plan{};
    pl.eb = eb;
    extra = 0;
    if (x <= 1 || y <= 1) return IPT_OK;
    Composed C;
    ipt_status_t s = valid_subword_eb(eb) ? resolve_subword(1, x * y, x, y, eb, C)
                                          : resolve_multiword(1, x * y, x, y, eb, 0, C);
    if (s != IPT_OK) return s;
    pl = C.e1.pl;
    pl.scratch = std::max(C.e1.cs.total, C.e2.cs.total) + C.rec_tmp;
    if (C.blocks) {
        extra = 1;
        if (!C.rec_tmp) pl.onchip = std::max(pl.onchip, static_cast<size_t>(C.rp.L) * C.rp.k * C.rec_w);
    }
    if (C.e2.batch) {
        extra += C.e2.pl.nlaunch;
        pl.onchip = std::max(pl.onchip, C.e2.pl.onchip);
    }
    return IPT_OK;
}

// Export -> P_{x,y} (reading C18): c2r(m,n,ROW) = P_{m,n}, c2r(m,n,COL) = P_{n,m};
// r2c is the inverse: r2c(m,n,ROW) = P_{n,m}, r2c(m,n,COL) = P_{m,n}.
bool perm_of(bool c2r, int64_t m, int64_t n, int layout, int64_t &x, int64_t &y) {
    if (layout != IPT_ROW_MAJOR && layout != IPT_COL_MAJOR) return false;
    const bool mn = (c2r == (layout == IPT_ROW_MAJOR));
    x = mn ? m : n;
    y = mn ? n : m;
    return true;
}

}  // namespace

cudaError_t ensure_kernel_attrs(const void *kern, size_t smem, bool nonportable_cluster) {
    static std::mutex mu;
    static std::unordered_map<std::string, size_t> smem_set;  // "kern@dev" -> limit set
    int dev = 0;
    cudaGetDevice(&dev);
    const std::string key = std::to_string(reinterpret_cast<uintptr_t>(kern)) + "@" + std::to_string(dev);
    std::lock_guard<std::mutex> lk(mu);
    auto it = smem_set.find(key);
    const size_t want = smem | (nonportable_cluster ? (size_t(1) << 62) : 0);
    if (it != smem_set.end() && (it->second & ~(size_t(1) << 62)) >= smem &&
        (!nonportable_cluster || (it->second >> 62))) return cudaSuccess;
    size_t have = it == smem_set.end() ? 0 : it->second;
    const size_t lim = std::max(smem, have & ~(size_t(1) << 62));
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(lim));
    if (e != cudaSuccess) return e;
    if (nonportable_cluster) {
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
    }
    smem_set[key] = lim | ((have | want) & (size_t(1) << 62));
    return cudaSuccess;
}

int cached_resident_blocks(const void *kern, int threads, size_t smem) {
    static std::mutex mu;
    static std::unordered_map<std::string, int> cache;
    int dev = 0;
    cudaGetDevice(&dev);
    const std::string key = std::to_string(reinterpret_cast<uintptr_t>(kern)) + "@" + std::to_string(dev) + "/" +
                            std::to_string(threads) + "/" + std::to_string(smem);
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find(key);
        if (it != cache.end()) return it->second;
    }
    int per_sm = 0, sms = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, smem) != cudaSuccess ||
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    std::lock_guard<std::mutex> lk(mu);
    cache[key] = per_sm * sms;
    return per_sm * sms;
}

}  // namespace ipt

using namespace ipt;

extern "C" {

ipt_status_t ipt_c2r(void *ptr, int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout, void *stream) {
    int64_t x, y;
    if (!perm_of(true, m, n, layout, x, y)) return IPT_ERR_INVALID_ARGUMENT;
    return run_perm_any(ptr, 1, -1, x, y, elem_bytes, stream);
}

ipt_status_t ipt_r2c(void *ptr, int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout, void *stream) {
    int64_t x, y;
    if (!perm_of(false, m, n, layout, x, y)) return IPT_ERR_INVALID_ARGUMENT;
    return run_perm_any(ptr, 1, -1, x, y, elem_bytes, stream);
}

ipt_status_t ipt_c2r_batched(void *base, int64_t batch, int64_t stride_elems, int64_t m, int64_t n, int elem_bytes,
                             ipt_layout_t layout, void *stream) {
    int64_t x, y;
    if (stride_elems < 0 || !perm_of(true, m, n, layout, x, y)) return IPT_ERR_INVALID_ARGUMENT;
    return run_perm_any(base, batch, stride_elems, x, y, elem_bytes, stream);
}

ipt_status_t ipt_r2c_batched(void *base, int64_t batch, int64_t stride_elems, int64_t m, int64_t n, int elem_bytes,
                             ipt_layout_t layout, void *stream) {
    int64_t x, y;
    if (stride_elems < 0 || !perm_of(false, m, n, layout, x, y)) return IPT_ERR_INVALID_ARGUMENT;
    return run_perm_any(base, batch, stride_elems, x, y, elem_bytes, stream);
}

static ipt_status_t run_host(bool c2r, void *host, void *dev, int64_t m, int64_t n, int elem_bytes,
                             ipt_layout_t layout, void *stream) {
    int64_t x, y;
    if (!host || !dev || elem_bytes <= 0 || !perm_of(c2r, m, n, layout, x, y)) return IPT_ERR_INVALID_ARGUMENT;
    if (m > 0 && n > (int64_t(1) << 62) / m / elem_bytes) return IPT_ERR_INVALID_ARGUMENT;
    const size_t bytes = static_cast<size_t>(m) * static_cast<size_t>(n) * static_cast<size_t>(elem_bytes);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    ipt_status_t s = check(cudaMemcpyAsync(dev, host, bytes, cudaMemcpyHostToDevice, st));
    if (s == IPT_OK) s = run_perm_any(dev, 1, -1, x, y, elem_bytes, stream);
    if (s == IPT_OK) s = check(cudaMemcpyAsync(host, dev, bytes, cudaMemcpyDeviceToHost, st));
    return s;
}

ipt_status_t ipt_c2r_host(void *host, void *dev, int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout,
                          void *stream) {
    return run_host(true, host, dev, m, n, elem_bytes, layout, stream);
}

ipt_status_t ipt_r2c_host(void *host, void *dev, int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout,
                          void *stream) {
    return run_host(false, host, dev, m, n, elem_bytes, layout, stream);
}

ipt_status_t ipt_aos_to_soa(void *ptr, int64_t count, int64_t fields, int field_bytes, void *stream) {
    return run_perm_any(ptr, 1, -1, count, fields, field_bytes, stream);  // P_{count,fields}
}

ipt_status_t ipt_soa_to_aos(void *ptr, int64_t count, int64_t fields, int field_bytes, void *stream) {
    return run_perm_any(ptr, 1, -1, fields, count, field_bytes, stream);  // P_{fields,count}
}

// Device scratch a one-matrix call of plan pl allocates (its CallScratch: counters, flags, wrap /
// boundary rows, side block; the skinny engine's tmp row and barrier word); composed element
// sizes keep their plan's figure.
static size_t call_scratch_bytes(const Plan &pl0, bool engine_step) {
    if (!engine_step) return pl0.scratch;
    Plan pl = pl0;
    CallScratch cs;
    prepare_call(pl, 1, cs);
    return std::max(pl0.scratch, cs.total);
}

ipt_status_t ipt_scratch_bytes(int64_t m, int64_t n, int elem_bytes, size_t *global_bytes, size_t *onchip_per_cta) {
    if (!(valid_eb(elem_bytes) || valid_multiword_eb(elem_bytes) || valid_subword_eb(elem_bytes)) || m < 0 || n < 0)
        return IPT_ERR_INVALID_ARGUMENT;
    Plan pl;
    ipt_status_t s;
    if (valid_eb(elem_bytes)) {
        s = engine_plan(m, n, elem_bytes, pl);
    } else {
        int64_t extra = 0;
        s = record_plan(m, n, elem_bytes, pl, extra);
    }
    if (s != IPT_OK) return s;
    if (global_bytes) *global_bytes = call_scratch_bytes(pl, valid_eb(elem_bytes));
    if (onchip_per_cta) *onchip_per_cta = pl.onchip;
    return IPT_OK;
}

ipt_status_t ipt_plan_info(int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout,
                           int64_t out[IPT_PLAN_INFO_FIELDS]) {
    int64_t x, y;
    if (!out || !(valid_eb(elem_bytes) || valid_multiword_eb(elem_bytes) || valid_subword_eb(elem_bytes)) ||
        m < 0 || n < 0 ||
        !perm_of(true, m, n, layout, x, y))
        return IPT_ERR_INVALID_ARGUMENT;
    Plan pl;
    int64_t extra_launches = 0;
    ipt_status_t s;
    if (valid_eb(elem_bytes)) {
        s = engine_plan(x, y, elem_bytes, pl);
    } else {  // multi-word element: plan of the engine step, launches of both
        s = record_plan(x, y, elem_bytes, pl, extra_launches);
    }
    if (s != IPT_OK) return s;
    out[0] = pl.engine;
    out[1] = pl.M;
    out[2] = pl.N;
    out[3] = pl.c;
    out[4] = pl.nlaunch + extra_launches;
    out[5] = pl.engine ? pl.shuf.p.G : 0;
    out[6] = pl.engine ? pl.shuf.p.W : 0;
    out[7] = static_cast<int64_t>(pl.onchip);
    out[8] = pl.engine ? pl.row.cl_K : 0;
    out[9] = static_cast<int64_t>(call_scratch_bytes(pl, valid_eb(elem_bytes)));
    return IPT_OK;
}

uint64_t ipt_launch_count(void) { return g_launches.load(); }

ipt_status_t ipt_debug_tile_copy(void *ptr, int64_t M, int64_t N, int elem_bytes, int tile_bytes, int cluster,
                                 int barrier, void *stream) {
    if (!valid_eb(elem_bytes) || M < 1 || N < 1 || M >= (1 << 29) || N >= (1 << 29) || cluster < 1 ||
        (tile_bytes != 128 && tile_bytes != 256 && tile_bytes != 512) ||
        !ptr || reinterpret_cast<uintptr_t>(ptr) % elem_bytes)
        return IPT_ERR_INVALID_ARGUMENT;
    const DevInfo dev = device_info();
    if (!dev.ok) return IPT_ERR_CUDA;
    ColParams p;
    std::memset(&p, 0, sizeof(p));
    p.base = static_cast<char *>(ptr);
    p.batch = 1;
    p.mat_stride_bytes = M * N * elem_bytes;
    p.M = static_cast<int32_t>(M);
    p.N = static_cast<int32_t>(N);
    p.c = p.a = p.b = 1;
    p.fd_c = p.fd_a = p.fd_b = make_fastdiv(1);
    p.fd_M = make_fastdiv(static_cast<uint32_t>(M));
    p.W = tile_bytes / elem_bytes;
    p.log2W = ilog2(p.W);
    p.ntiles = static_cast<int32_t>((N + p.W - 1) / p.W);
    p.B = static_cast<int32_t>((M + cluster - 1) / cluster);
    if (p.B > col_max_band(p.W)) return IPT_ERR_UNSUPPORTED;
    p.G = static_cast<int32_t>((M + p.B - 1) / p.B);
    p.rot_sign = barrier ? 1 : 0;
    const bool pipe = env_int("IPT_COL_PIPE", 1) != 0;
    p.pipe = pipe ? 1 : 0;
    p.nbuf = pipe ? std::min(std::max(env_int("IPT_COL_NBUF", 2), 2), col_max_bufs()) : 1;
    const size_t smem = col_smem_bytes(p.B, p.W, elem_bytes, p.nbuf);
    if (smem > static_cast<size_t>(dev.smem_optin)) return IPT_ERR_UNSUPPORTED;
    p.threads = pipe ? col_block_threads() : static_cast<int>(env_int("IPT_COL_THREADS", 256));
    p.resident = col_resident_ctas(COL_COPY, elem_bytes, tile_bytes, smem, pipe, p.threads);
    if (p.resident < p.G) return IPT_ERR_UNSUPPORTED;
    finish_col(p, 1);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    char *ctr = nullptr;
    ipt_status_t s = pool_alloc(&ctr, kCtrBytes, st);
    if (s != IPT_OK) return s;
    s = check(cudaMemsetAsync(ctr, 0, kCtrBytes, st));
    p.ctr = reinterpret_cast<unsigned int *>(ctr);
    p.ticket = 1;
    if (s == IPT_OK) s = check(launch_col(p, COL_COPY, elem_bytes, st, smem));
    cudaFreeAsync(ctr, st);
    return s;
}

void ipt_profile_enable(int on) { g_prof_on.store(on ? 1 : 0); }

int64_t ipt_profile_read(int64_t *launches, double *ms, double *bytes) {
    std::vector<ProfRec> recs;
    {
        std::lock_guard<std::mutex> lk(g_prof_mu);
        recs.swap(g_prof);
    }
    for (int k = 0; k < IPT_PROFILE_KINDS; ++k) {
        if (launches) launches[k] = 0;
        if (ms) ms[k] = 0;
        if (bytes) bytes[k] = 0;
    }
    bool ok = true;
    for (ProfRec &r : recs) {
        float t = 0;
        if (cudaEventSynchronize(r.stop) != cudaSuccess || cudaEventElapsedTime(&t, r.start, r.stop) != cudaSuccess)
            ok = false;
        if (r.kind >= 0 && r.kind < IPT_PROFILE_KINDS) {
            if (launches) launches[r.kind] += 1;
            if (ms) ms[r.kind] += t;
            if (bytes) bytes[r.kind] += r.bytes;
        }
        cudaEventDestroy(r.start);
        cudaEventDestroy(r.stop);
    }
    if (!ok) {
        cudaGetLastError();
        return -1;
    }
    return static_cast<int64_t>(recs.size());
}

const char *ipt_status_string(ipt_status_t s) {
    switch (s) {
        case IPT_OK: return "IPT_OK";
        case IPT_ERR_INVALID_ARGUMENT: return "IPT_ERR_INVALID_ARGUMENT";
        case IPT_ERR_UNSUPPORTED: return "IPT_ERR_UNSUPPORTED";
        case IPT_ERR_OUT_OF_MEMORY: return "IPT_ERR_OUT_OF_MEMORY";
        case IPT_ERR_CUDA: return "IPT_ERR_CUDA";
        default: return "IPT_UNKNOWN_STATUS";
    }
}

}  // extern "C"
