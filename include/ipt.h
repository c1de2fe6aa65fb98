/*
 * include/ipt.h -- C ABI of the B200 (sm_100a) decomposed in-place transpose.
 *
 * Method: Catanzaro, Keller, Garland, "A Decomposition for In-place Matrix
 * Transposition", PPoPP'14.  Citations are PAPER.md lines + equation/section.
 *
 * Every entry point is asynchronous on `stream` (a cudaStream_t of the current device,
 * passed as void* so that this header needs no CUDA include; NULL = legacy default
 * stream).  Arguments are validated, and every step of the call planned (including the
 * UNSUPPORTED checks of composed element sizes), synchronously before anything is
 * enqueued; such an error leaves the buffer untouched.  No entry point allocates device
 * memory that outlives the call, throws, or synchronises the stream.  All entry points are
 * thread-safe and reentrant: every call owns one stream-ordered scratch allocation (its
 * counters, flags and boundary rows), so concurrent calls from any threads on any streams
 * (cudaStreamPerThread included) share no state.
 *
 * Forward progress: no kernel relies on its CTAs being co-resident or dispatched in index
 * order.  Cross-CTA waits (the column pass's lagged-layout counters, the fused rotation's
 * row flags) only ever target work units with a smaller dispatch ticket, taken by a CTA
 * already running; passes whose CTAs must be co-resident (per-tile group barriers: the
 * separate rotation pass for gcd > 32 and unlagged shuffles) are cooperative launches, which
 * fail with IPT_ERR_CUDA instead of hanging when the GPU cannot host the whole grid.
 *
 * Memory: `ptr` is caller-owned device memory on the current device, aligned to
 * elem_bytes (16-byte alignment is NOT required).  The caller must not read or write it
 * until the stream reaches the end of the call.  The operation is not atomic: if a
 * launch fails mid-sequence (IPT_ERR_CUDA) the buffer content is unspecified.
 *
 * Element size: elem_bytes in {4, 8, 16} natively (the engine's passes); 1, 2 and any
 * other multiple of 4 up to 4096 by composition (below).  Elements are opaque words (bit-exact moves,
 * no floating-point semantics; NaN payloads, -0.0 and subnormals are preserved).
 *
 * Sub-word elements: elem_bytes in {1, 2}, `ptr` 4-byte aligned.  g = 4 / elem_bytes
 * elements share one 4-byte engine word: with P_{x,y} the export's permutation, y % g == 0
 * runs P_{x,y/g} on words and then splits each row of x g-tuples into g rows; x % g == 0
 * merges each group of g rows into y g-tuples and runs P_{x/g,y} on words (when both are
 * possible, the one with the shorter blocks: split if x <= y) (one
 * record-block pass + one engine call; the buffer moves twice).  IPT_ERR_UNSUPPORTED when
 * neither x nor y is a multiple of g, when a batch stride is not a multiple of g, or when
 * a block of 4*min-side bytes exceeds the record pass's scratch budget.
 *
 * Multi-word elements (records): elem_bytes = k*w for any multiple of 4 up to 4096 that is
 * not 4, 8 or 16 (12, 24, 32, 48, 64 B ...).  `ptr` then needs 4-byte alignment only; w is
 * the largest of 16, 8, 4 dividing both elem_bytes and the address.  Such a call runs two
 * word-level permutations (the paper's passes move opaque words of any size,
 * PAPER.md:1037, :1085), so it moves the buffer twice.  With L = min(x, y) records
 * (P_{x,y} = the export's permutation): x <= y runs P_{x,y*k} on w-byte words, then P_{k,x}
 * on each of the y k-by-x blocks (one record-block pass); x > y first splits each row of y
 * records into k-by-y words (P_{y,k}, same pass), then runs P_{x*k,y} on words.  A block
 * is staged in shared memory when L*elem_bytes <= 220 KiB, else in a per-CTA slot of
 * stream-ordered global scratch (one slot per SM or more, <= 1 GiB in total); beyond that
 * both steps run on the engine (a strided batch, stride_elems > m*n, then runs the second
 * step once per matrix).
 */
#ifndef IPT_H_
#define IPT_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    IPT_ROW_MAJOR = 0, /* element (i, j) of the m x n matrix at offset i*n + j (Eq. 1, :85)  */
    IPT_COL_MAJOR = 1  /* element (i, j) of the m x n matrix at offset i + j*m (Eq. 4, :99)  */
} ipt_layout_t;

typedef enum {
    IPT_OK = 0,
    IPT_ERR_INVALID_ARGUMENT = 1, /* negative dims, bad elem_bytes/layout, NULL or misaligned
                                     ptr (to elem_bytes for 4/8/16, else to 4), stride < m*n,
                                     size overflow; buffer untouched                         */
    IPT_ERR_UNSUPPORTED = 2,      /* shape beyond the implemented on-chip staging limits, or
                                     the device is not sm_100; buffer untouched              */
    IPT_ERR_OUT_OF_MEMORY = 3,    /* scratch allocation failed; buffer untouched            */
    IPT_ERR_CUDA = 4              /* a launch failed; buffer contents unspecified            */
} ipt_status_t;

/*
 * ipt_c2r -- in-place transpose.
 *   In:  an m x n matrix stored in `layout` at ptr.
 *   Out: its n x m transpose, stored in the same layout, in the same memory.
 * Row-major input is the paper's C2R (Theorem 1: "The C2R transpose
 * implements transposition for row-major arrays"); column-major input swaps m and n
 * (Theorem 2, :227-255).  Internally the library runs the decomposed algorithm
 * (Algorithm 1, :569-599; gather forms §4.2-4.3, :669-743) on whichever engine the
 * heuristic of :959 selects (C2R if the array has more rows than columns, else R2C; both
 * induce the same permutation, Theorem 2/7).  Passes: [column rotation if gcd > 1]
 * (Eq. 23), row shuffle (Eq. 31 / 24), column shuffle (Eq. 26 = p_j o q, Eqs. 32-33).
 * Auxiliary space: O(max(m, n)) elements per worker (Theorem 6, :605), on chip; see
 * ipt_scratch_bytes.  m or n in {0, 1} is the identity: IPT_OK, nothing enqueued.
 */
ipt_status_t ipt_c2r(void *ptr, int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout,
                     void *stream);

/*
 * ipt_r2c -- the exact inverse of ipt_c2r with the same arguments ("The R2C
 * and C2R transposes are inverses of each other"; :603).  In: the n x m matrix produced
 * by ipt_c2r(ptr, m, n, elem_bytes, layout); out: the original m x n matrix.
 */
ipt_status_t ipt_r2c(void *ptr, int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout,
                     void *stream);

/*
 * Batched variants: `batch` independent matrices, matrix k at
 * (char*)base + k * stride_elems * elem_bytes, stride_elems >= m*n.  One plan, one launch
 * per pass for the whole batch (the paper's rows and columns are independent units,
 * Theorem 4, :479; batches add a third independent axis).  Matrices must not overlap.
 */
ipt_status_t ipt_c2r_batched(void *base, int64_t batch, int64_t stride_elems, int64_t m,
                             int64_t n, int elem_bytes, ipt_layout_t layout, void *stream);
ipt_status_t ipt_r2c_batched(void *base, int64_t batch, int64_t stride_elems, int64_t m,
                             int64_t n, int elem_bytes, ipt_layout_t layout, void *stream);

/*
 * Host-buffer variants (the end-to-end call): the m x n matrix lives in HOST memory at
 * `host` (pinned for asynchronous copies; pageable memory works but the copies are then
 * synchronous); `dev` is caller-owned device memory of at least m*n*elem_bytes bytes.
 * Stream-ordered on `stream`: copy host -> dev, ipt_c2r / ipt_r2c on dev (same semantics
 * and arguments as above), copy dev -> host.  On return nothing has necessarily run yet;
 * synchronise the stream before reading `host`.  Consecutive calls on several streams with their own
 * device buffers overlap one call's device->host copy with the next call's host->device
 * copy (the two directions of the host link).  Errors: IPT_ERR_INVALID_ARGUMENT for a null
 * host/dev pointer or the arguments ipt_c2r rejects; other codes as ipt_c2r.  On any error
 * the host buffer is unchanged (no device->host copy is enqueued); dev is unspecified.
 */
ipt_status_t ipt_c2r_host(void *host, void *dev, int64_t m, int64_t n, int elem_bytes,
                          ipt_layout_t layout, void *stream);
ipt_status_t ipt_r2c_host(void *host, void *dev, int64_t m, int64_t n, int elem_bytes,
                          ipt_layout_t layout, void *stream);

/*
 * Skinny AoS <-> SoA conversion (§6.1).  An Array of Structures of
 * `count` structs, each of `fields` fields of field_bytes bytes, is a row-major
 * count x fields array; ipt_aos_to_soa transposes it in place into `fields` arrays of
 * `count` (the Structure of Arrays).  ipt_soa_to_aos is the exact inverse.  Equivalent to
 * ipt_c2r / ipt_r2c(ptr, count, fields, field_bytes, IPT_ROW_MAJOR, stream), routed to the
 * specialised skinny engine when fields <= 32.
 */
ipt_status_t ipt_aos_to_soa(void *ptr, int64_t count, int64_t fields, int field_bytes,
                            void *stream);
ipt_status_t ipt_soa_to_aos(void *ptr, int64_t count, int64_t fields, int field_bytes,
                            void *stream);

/*
 * Auxiliary-space statement for ipt_c2r(m, n, elem_bytes, ...) (Theorem 6, PAPER.md:605:
 * O(max(m, n)) auxiliary space).  *global_bytes: device scratch the call allocates
 * (stream-ordered, freed before the call's work completes) for one matrix: the column-pass
 * counters (16 KB per column pass), the side block of the lagged column-tile layout (M rows x
 * 8 tiles of 128 B, M = max(m, n)), and with a fused rotation either one flag per row plus
 * gcd(m, n) - 1 wrapped rows or gcd(m, n) - 1 boundary rows per chunk of >= 8 (gcd - 1) rows;
 * the skinny engine one row of the long dimension (+ 256 B).  Batched calls scale it by the
 * batch (the side block capped at max(256 MiB, 1/8 of the data)).  *onchip_per_cta: the largest shared-memory staging buffer
 * of any launched CTA.  Multi-word elem_bytes: the larger of the two word-level steps
 * (words as wide as a 16-byte-aligned base allows).  Either pointer may be NULL.
 */
ipt_status_t ipt_scratch_bytes(int64_t m, int64_t n, int elem_bytes, size_t *global_bytes,
                               size_t *onchip_per_cta);

/* Static description of a status code. */
const char *ipt_status_string(ipt_status_t s);

/*
 * Introspection for tests and benchmarks (no side effects).  Fills `out` with the plan
 * the library would run for ipt_c2r(m, n, elem_bytes, layout): out[0] engine (0 none,
 * 1 C2R, 2 R2C, 3 skinny), out[1] M (engine rows), out[2] N (engine columns), out[3] c =
 * gcd(M, N), out[4] number of kernel launches, out[5] column-tile cluster size, out[6]
 * column-tile width in elements, out[7] largest on-chip staging bytes per CTA, out[8]
 * CTAs per row of the row pass (0: one CTA per row; K > 0: a K-CTA cluster sharing the
 * row through distributed shared memory, for rows longer than one CTA's shared memory),
 * out[9] global scratch bytes.  Multi-word elem_bytes: out[0..3], out[5..9] describe the
 * engine's word-level step; out[4] counts the launches of both steps (one matrix).
 * Returns IPT_ERR_UNSUPPORTED for shapes beyond limits.
 */
#define IPT_PLAN_INFO_FIELDS 10
ipt_status_t ipt_plan_info(int64_t m, int64_t n, int elem_bytes, ipt_layout_t layout,
                           int64_t out[IPT_PLAN_INFO_FIELDS]);

/* Number of kernel launches this library has enqueued since load (all threads). */
uint64_t ipt_launch_count(void);

/*
 * Per-kernel timing for benchmarks.  While enabled (process-wide), every launch is
 * bracketed by two CUDA events recorded on the launch's own stream.  ipt_profile_read
 * waits for those events and returns, per kernel kind k (0 row shuffle, 1 column
 * shuffle, 2 column rotation, 3 skinny pass), launches[k], the summed device time ms[k]
 * and the summed ALGORITHMIC bytes bytes[k] (what the pass must move: one read and one
 * write of every element it permutes, Eq. 37's 2mns per full pass);
 * then clears the record.  Arrays have IPT_PROFILE_KINDS entries.  Returns the number of
 * launches read, or -1 on a CUDA error.
 */
#define IPT_PROFILE_KINDS 8
void ipt_profile_enable(int on);
int64_t ipt_profile_read(int64_t *launches, double *ms, double *bytes);

#ifdef __cplusplus
}
#endif

#endif /* IPT_H_ */
