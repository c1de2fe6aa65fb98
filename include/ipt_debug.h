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
 * kernel roofline).  tile_bytes in {32, 64, 128}; 1 <= cluster <= co-resident CTAs.  Asynchronous on
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

#ifdef __cplusplus
}
#endif

#endif /* IPT_DEBUG_H_ */
