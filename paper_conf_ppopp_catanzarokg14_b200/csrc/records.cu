// Record blocks: the local step of a multi-word-element transpose.
//
// An element of k words (a record of eb = k*w bytes) is transposed with one word-level
// engine call plus this pass over independent blocks of L records (api.cu run_perm_any):
//   split: one block = L x k words (L records)     -> k x L words (word v of every record);
//   merge: one block = k x L words                 -> L x k words (L records).
// Sub-word elements (1 or 2 bytes) use the same pass with k = 4 / eb elements per 4-byte
// engine word (api.cu run_perm_subword).
// These are the P_{L,k} / P_{k,L} of the paper's Theorem 1 buffer form
// on one block per CTA at a time: the block is staged whole with coalesced loads, then
// written back coalesced in its new order, so each byte is read and written once (2*L*eb
// bytes per block, HBM bound).  Blocks up to kRecordSmemMax are staged in shared memory;
// longer ones in a per-CTA slot of a global scratch buffer sized to stay L2-resident
// (Theorem 6's O(max(m, n)) auxiliary space per worker).
#include "common.cuh"
#include "plan.h"

namespace ipt {

namespace {

constexpr int kRecThreads = 512;

// G x G transpose of sub-word elements held in G 32-bit words (G = 4 / W): out[e] element v
// = in[v] element e.  1-byte: a 4x4 byte transpose in six byte permutes; 2-byte: two.
template <int W>
__device__ __forceinline__ void tuple_transpose(const uint32_t (&in)[4 / W], uint32_t (&out)[4 / W]) {
    if constexpr (W == 1) {
        const uint32_t t0 = __byte_perm(in[0], in[1], 0x5140), t1 = __byte_perm(in[0], in[1], 0x7362);
        const uint32_t t2 = __byte_perm(in[2], in[3], 0x5140), t3 = __byte_perm(in[2], in[3], 0x7362);
        out[0] = __byte_perm(t0, t2, 0x5410);
        out[1] = __byte_perm(t0, t2, 0x7632);
        out[2] = __byte_perm(t1, t3, 0x5410);
        out[3] = __byte_perm(t1, t3, 0x7632);
    } else {
        out[0] = __byte_perm(in[0], in[1], 0x5410);
        out[1] = __byte_perm(in[0], in[1], 0x7632);
    }
}

template <int W, bool GLOBAL>
__global__ void __launch_bounds__(kRecThreads) record_block_kernel(RecordParams p) {
    using T = typename Word<W>::T;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    // GLOBAL: this CTA's slot of the scratch buffer (plain loads: written by this CTA,
    // made visible to its threads by __syncthreads).
    T *s = GLOBAL ? reinterpret_cast<T *>(p.tmp + static_cast<int64_t>(blockIdx.x) * p.L * p.k * W)
                  : reinterpret_cast<T *>(smem_raw);
    const uint32_t L = p.L, k = p.k, n = p.L * p.k;
    const FastDiv fk = p.fd_k;
    for (int64_t blk = blockIdx.x; blk < p.nblocks; blk += gridDim.x) {
        const int64_t b = blk / p.per_mat, j = blk - b * p.per_mat;
        T *g = reinterpret_cast<T *>(p.base + b * p.mat_stride_bytes + j * p.blk_stride_bytes);
        if constexpr (W < 4) {
            // Sub-word elements (k = G = 4 / W): the block is L whole 32-bit words.  With
            // L % G == 0 every output row is word-aligned too, so thread c moves one G x G
            // tile: G words in, G words out, transposed in registers.
            constexpr uint32_t G = 4 / W;
            uint32_t *g32 = reinterpret_cast<uint32_t *>(g), *s32 = reinterpret_cast<uint32_t *>(s);
            for (uint32_t t = threadIdx.x; t < L; t += kRecThreads) s32[t] = g32[t];
            __syncthreads();
            if (L % G == 0) {
                const uint32_t wpr = L / G;  // words per row of G elements' worth
                for (uint32_t c = threadIdx.x; c < wpr; c += kRecThreads) {
                    uint32_t in[G], out[G];
                    if (p.split) {  // tuples c*G .. c*G+G-1 -> word c of rows 0..G-1
#pragma unroll
                        for (uint32_t e = 0; e < G; ++e) in[e] = s32[c * G + e];
                        tuple_transpose<W>(in, out);
#pragma unroll
                        for (uint32_t v = 0; v < G; ++v) g32[v * wpr + c] = out[v];
                    } else {        // word c of rows 0..G-1 -> tuples c*G .. c*G+G-1
#pragma unroll
                        for (uint32_t v = 0; v < G; ++v) in[v] = s32[v * wpr + c];
                        tuple_transpose<W>(in, out);
#pragma unroll
                        for (uint32_t e = 0; e < G; ++e) g32[c * G + e] = out[e];
                    }
                }
            } else {
                // Ragged rows (L % G != 0): still whole output words; each of the word's G
                // elements is located on its own (split: row v = o / L; merge: o / G).
                using E = typename Word<W>::T;
                const E *se = reinterpret_cast<const E *>(s32);
                for (uint32_t t = threadIdx.x; t < L; t += kRecThreads) {
                    uint32_t word = 0;
#pragma unroll
                    for (uint32_t e = 0; e < G; ++e) {
                        const uint32_t o = t * G + e;
                        uint32_t src;
                        if (p.split) {
                            const uint32_t v = fdiv(o, p.fd_L);
                            src = (o - v * L) * G + v;
                        } else {
                            src = (o % G) * L + o / G;
                        }
                        word |= static_cast<uint32_t>(se[src]) << (8 * W * e);
                    }
                    g32[t] = word;
                }
            }
            __syncthreads();
            continue;
        } else {
            for (uint32_t t = threadIdx.x; t < n; t += kRecThreads) s[t] = g[t];
            __syncthreads();
        }
        if (p.split) {  // L x k -> k x L: out[v*L + i] = in[i*k + v]
            for (uint32_t v = 0; v < k; ++v)
                for (uint32_t i = threadIdx.x; i < L; i += kRecThreads) g[v * L + i] = s[i * k + v];
        } else {        // k x L -> L x k: out[i*k + v] = in[v*L + i]
            for (uint32_t o = threadIdx.x; o < n; o += kRecThreads) {
                const uint32_t i = fdiv(o, fk), v = o - i * k;
                g[o] = s[v * L + i];
            }
        }
        __syncthreads();  // the buffer is refilled by the next block
    }
}

// Short blocks (<= kChunkBlockMax bytes; e.g. AoS<->SoA with a few fields): one CTA would
// idle on a tiny block per barrier pair, so each CTA stages a chunk of consecutive blocks of
// one matrix (blocks are contiguous: blk_stride = L*k*W) and permutes every element of the
// chunk, locating it by strength-reduced divisions.
constexpr uint32_t kChunkBlockMax = 4096, kChunkBytes = 32768;

template <int W>
__global__ void __launch_bounds__(kRecThreads) record_chunk_kernel(RecordParams p, uint32_t chunk, FastDiv fd_n,
                                                                   FastDiv fd_L) {
    using T = typename Word<W>::T;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T *s = reinterpret_cast<T *>(smem_raw);
    const uint32_t L = p.L, k = p.k, n = p.L * p.k;
    const int64_t cpm = (p.per_mat + chunk - 1) / chunk, items = p.nblocks / p.per_mat * cpm;
    for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
        const int64_t b = it / cpm, j0 = (it - b * cpm) * chunk;
        const uint32_t nb = static_cast<uint32_t>(p.per_mat - j0 < chunk ? p.per_mat - j0 : chunk);
        T *g = reinterpret_cast<T *>(p.base + b * p.mat_stride_bytes + j0 * p.blk_stride_bytes);
        const uint32_t tot = nb * n;
        for (uint32_t t = threadIdx.x; t < tot; t += kRecThreads) s[t] = g[t];
        __syncthreads();
        for (uint32_t t = threadIdx.x; t < tot; t += kRecThreads) {
            const uint32_t blk = fdiv(t, fd_n), r = t - blk * n;
            uint32_t src;
            if (p.split) {  // out[v*L + i] = in[i*k + v]
                const uint32_t v = fdiv(r, fd_L), i = r - v * L;
                src = i * k + v;
            } else {        // out[i*k + v] = in[v*L + i]
                const uint32_t i = fdiv(r, p.fd_k), v = r - i * k;
                src = v * L + i;
            }
            g[t] = s[blk * n + src];
        }
        __syncthreads();  // the buffer is refilled by the next chunk
    }
}

template <int W>
cudaError_t launch_w(const RecordParams &p, cudaStream_t st) {
    const size_t blk_bytes = static_cast<size_t>(p.L) * p.k * W;
    if (!p.tmp && blk_bytes <= kChunkBlockMax && p.per_mat > 1) {
        const uint32_t chunk = static_cast<uint32_t>(kChunkBytes / blk_bytes);
        const size_t smem = chunk * blk_bytes;
        auto kern = record_chunk_kernel<W>;
        cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
        if (e != cudaSuccess) return e;
        const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kRecThreads, smem);
        if (resident < 1) return cudaErrorInvalidConfiguration;
        const int64_t items = p.nblocks / p.per_mat * ((p.per_mat + chunk - 1) / chunk);
        const int64_t grid = items < resident ? items : resident;
        kern<<<static_cast<unsigned>(grid), kRecThreads, smem, st>>>(
            p, chunk, make_fastdiv(p.L * p.k), make_fastdiv(p.L));
        return cudaGetLastError();
    }
    if (p.tmp) {
        record_block_kernel<W, true><<<p.grid, kRecThreads, 0, st>>>(p);
        return cudaGetLastError();
    }
    const size_t smem = static_cast<size_t>(p.L) * p.k * W;
    auto kern = record_block_kernel<W, false>;
    cudaError_t e = ensure_kernel_attrs(reinterpret_cast<const void *>(kern), smem, false);
    if (e != cudaSuccess) return e;
    const int resident = cached_resident_blocks(reinterpret_cast<const void *>(kern), kRecThreads, smem);
    if (resident < 1) return cudaErrorInvalidConfiguration;
    const int64_t grid = p.nblocks < resident ? p.nblocks : resident;
    kern<<<static_cast<unsigned>(grid), kRecThreads, smem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_record_blocks(const RecordParams &p, int w, cudaStream_t st) {
    switch (w) {
        case 1: return launch_w<1>(p, st);
        case 2: return launch_w<2>(p, st);
        case 4: return launch_w<4>(p, st);
        case 8: return launch_w<8>(p, st);
        case 16: return launch_w<16>(p, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace ipt
