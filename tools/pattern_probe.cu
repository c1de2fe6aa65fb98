// Standalone DRAM access-pattern probe (measurement tool, not product code).
// Copies an M x N (bytes: M rows of R bytes) array with different traversal orders and
// reports GB/s = 2*M*R / t:
//   contiguous      : 16-byte vector grid-stride copy
//   tile<TW>        : one CTA per (column tile of TW bytes, band of rows), warps read
//                     TW-byte sub-rows at stride R and write them back (no smem)
//   tile<TW>_staged : same, but the CTA first loads its whole band into smem (cp.async),
//                     __syncthreads, then stores (the column kernel's phase structure)
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o pattern_probe tools/pattern_probe.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void copy_contig(const uint4 *__restrict__ a, uint4 *__restrict__ b, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        b[i] = a[i];
}

// TW bytes per sub-row, lanes per row = TW/16; warp covers 32/(TW/16) rows per instruction.
template <int TW>
__global__ void copy_tile(const char *__restrict__ a, char *__restrict__ b, int M, int R, int band) {
    constexpr int LPR = TW / 16;
    const int ntile = R / TW;
    const int tile = blockIdx.x % ntile;
    const int bandi = blockIdx.x / ntile;
    const int r0 = bandi * band, r1 = min(M, r0 + band);
    const int sub = threadIdx.x % LPR;
    for (int r = r0 + threadIdx.x / LPR; r < r1; r += blockDim.x / LPR) {
        size_t off = (size_t)r * R + (size_t)tile * TW + sub * 16;
        *(uint4 *)(b + off) = *(const uint4 *)(a + off);
    }
}

template <int TW>
__global__ void copy_tile_staged(char *a, int M, int R, int band, int tile_major) {
    extern __shared__ __align__(16) unsigned char sm[];
    constexpr int LPR = TW / 16;
    const int ntile = R / TW;
    const int nband = (M + band - 1) / band;
    const int tile = tile_major ? blockIdx.x / nband : blockIdx.x % ntile;
    const int bandi = tile_major ? blockIdx.x % nband : blockIdx.x / ntile;
    const int r0 = bandi * band, r1 = min(M, r0 + band);
    const int sub = threadIdx.x % LPR;
    uint32_t s = (uint32_t)__cvta_generic_to_shared(sm);
    for (int r = r0 + threadIdx.x / LPR; r < r1; r += blockDim.x / LPR) {
        size_t off = (size_t)r * R + (size_t)tile * TW + sub * 16;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s + (uint32_t)((r - r0) * TW + sub * 16)),
                     "l"(a + off));
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
    __syncthreads();
    for (int r = r0 + threadIdx.x / LPR; r < r1; r += blockDim.x / LPR) {
        size_t off = (size_t)r * R + (size_t)tile * TW + sub * 16;
        *(uint4 *)(a + off) = *(const uint4 *)(sm + (r - r0) * TW + sub * 16);
    }
}

static float timeit(void (*f)(void *), void *arg, char *flush, size_t fl) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e9;
    for (int k = 0; k < 5; ++k) {
        cudaMemset(flush, k, fl);
        cudaEventRecord(e0);
        f(arg);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (k > 0 && ms < best) best = ms;
    }
    return best;
}

struct Args {
    char *a, *b;
    int M, R, band, grid, threads;
    size_t smem;
};
static Args G;

template <int TW> void run_tile(void *) {
    int ntile = G.R / TW, nb = (G.M + G.band - 1) / G.band;
    copy_tile<TW><<<ntile * nb, G.threads>>>(G.a, G.b, G.M, G.R, G.band);
}
template <int TW> void run_tile_staged(void *) {
    int ntile = G.R / TW, nb = (G.M + G.band - 1) / G.band;
    copy_tile_staged<TW><<<ntile * nb, G.threads, (size_t)G.band * TW>>>(G.a, G.M, G.R, G.band, G.grid);
}
void run_contig(void *) { copy_contig<<<148 * 8, 512>>>((const uint4 *)G.a, (uint4 *)G.b, (size_t)G.M * G.R / 16); }

int main(int argc, char **argv) {
    int M = argc > 1 ? atoi(argv[1]) : 17226;
    int R = argc > 2 ? atoi(argv[2]) : 6052 * 4;
    const int align = argc > 3 ? atoi(argv[3]) : 128;
    R = R / align * align;  // row pitch alignment (128: line-aligned tiles; 16: misaligned rows)
    size_t bytes = (size_t)M * R;
    cudaMalloc(&G.a, bytes);
    cudaMalloc(&G.b, bytes);
    cudaMemset(G.a, 1, bytes);
    char *flush;
    size_t fl = 256u << 20;
    cudaMalloc(&flush, fl);
    G.M = M;
    G.R = R;
    G.threads = 512;
    G.grid = argc > 4 ? atoi(argv[4]) : 0;  // 1: tile-major block order
    float t = timeit(run_contig, nullptr, flush, fl);
    printf("{\"what\":\"contiguous\",\"GBps\":%.1f}\n", 2.0 * bytes / t / 1e6);
    // staged copies at a fixed shared-memory budget per CTA (the column kernel's unit size)
    for (size_t sm : {size_t(27) << 10, size_t(54) << 10, size_t(108) << 10}) {
        for (int tw : {128, 256, 512}) {
            G.band = (int)(sm / tw);
            void (*f)(void *) = tw == 128 ? run_tile_staged<128> : tw == 256 ? run_tile_staged<256> : run_tile_staged<512>;
            const void *k = tw == 128 ? (const void *)copy_tile_staged<128>
                            : tw == 256 ? (const void *)copy_tile_staged<256> : (const void *)copy_tile_staged<512>;
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            t = timeit(f, nullptr, flush, fl);
            printf("{\"what\":\"tile%d_staged\",\"band\":%d,\"smem\":%zu,\"GBps\":%.1f}\n", tw, G.band, sm,
                   2.0 * bytes / t / 1e6);
        }
    }
    for (int band : {256, 512}) {
        G.band = band;
        t = timeit(run_tile<128>, nullptr, flush, fl);
        printf("{\"what\":\"tile128\",\"band\":%d,\"GBps\":%.1f}\n", band, 2.0 * bytes / t / 1e6);
        t = timeit(run_tile<256>, nullptr, flush, fl);
        printf("{\"what\":\"tile256\",\"band\":%d,\"GBps\":%.1f}\n", band, 2.0 * bytes / t / 1e6);
        t = timeit(run_tile<512>, nullptr, flush, fl);
        printf("{\"what\":\"tile512\",\"band\":%d,\"GBps\":%.1f}\n", band, 2.0 * bytes / t / 1e6);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) printf("err %s\n", cudaGetErrorString(e));
    return 0;
}
