/*
 * include/ipt_debug.h -- measurement hooks of libipt.so (not part of the transpose API).
 *
 * ipt_debug_tile_copy: run the column-tile kernel in identity mode on an M x N row-major
 * array (out[i][j] = in[i][j]): every M x (tile_bytes / elem_bytes) column tile is staged
 * on chip by a group of `cluster` CTAs (bands of ceil(M / cluster) rows) and written back
 * unchanged.  barrier = 1 keeps the group barrier of the real column passes, barrier = 0
 * drops it.  It isolates the
 * cost of the tile access pattern (strided tile_bytes-wide sub-rows) and of the cluster
 * synchronisation from the index arithmetic of the permutations (column
 * kernel roofline).  tile_bytes in {128, 256, 512}; 1 <= cluster <= co-resident CTAs.  Asynchronous on
 * `stream`; the buffer content is unchanged on success.
 */
#ifndef IPT_DEBUG_H_
#define IPT_DEBUG_H_

#include <stdint.h>

#include "ipt.h"

#ifdef __cplusplus
extern "C" {
#endif

ipt_status_t ipt_debug_tile_copy(void *ptr, int64_t M, int64_t N, int elem_bytes, int tile_bytes, int cluster,
                                 int barrier, void *stream);

/*
 * Consumer kernels of include/ipt/aos.cuh (§6.2, Figs. 8-10; SURVEY §8 row a6,
 * BASELINE config 4) over `count` structs of `words` 4-byte words (1..32), contiguous:
 *   ipt_debug_aos_copy: dst[k] = src[k];  ipt_debug_aos_fill: word i of dst[k] = k*words + i.
 * variant: IPT_AOS_DIRECT (compiler-generated per-lane struct access), IPT_AOS_VECTOR
 * (widest native vector dividing the struct), IPT_AOS_COALESCED (coalesced_ptr<T>).
 * ipt_debug_warp_load_dump: per 32-struct chunk, dump[lane*words + k] = register k of lane
 *   after warp_load_aos (must equal the chunk).  ipt_debug_warp_store: lane l's registers
 *   taken per lane from regs[l*words + k], stored with warp_store_aos (dst must equal regs).
 * nchunks counts chunks of 32 structs.
 */
#define IPT_AOS_DIRECT 0
#define IPT_AOS_VECTOR 1
#define IPT_AOS_COALESCED 2
ipt_status_t ipt_debug_aos_copy(const void *src, void *dst, int64_t count, int words, int variant, void *stream);
ipt_status_t ipt_debug_aos_fill(void *dst, int64_t count, int words, int variant, void *stream);
ipt_status_t ipt_debug_warp_load_dump(const void *src, void *dump, int64_t nchunks, int words, void *stream);
/*
 * Random-access consumers (SURVEY §8 row f1; PAPER.md :1087, :1099, Fig. 9) of
 * warp_gather_aos / warp_scatter_aos: ipt_debug_aos_gather: dst[k] = src[idx[k]];
 * ipt_debug_aos_scatter: dst[idx[k]] = src[k] (idx a permutation for a defined result).
 * `count` structs of `words` words; idx[k] < number of structs of src (gather) / dst
 * (scatter); variants as above (COALESCED = the cooperative helpers on whole warps).
 */
ipt_status_t ipt_debug_aos_gather(const void *src, const uint32_t *idx, void *dst, int64_t count, int words,
                                  int variant, void *stream);
ipt_status_t ipt_debug_aos_scatter(const void *src, const uint32_t *idx, void *dst, int64_t count, int words,
                                   int variant, void *stream);
ipt_status_t ipt_debug_warp_store(const void *regs, void *dst, int64_t nchunks, int words, void *stream);

#ifdef __cplusplus
}
#endif

#endif /* IPT_DEBUG_H_ */
