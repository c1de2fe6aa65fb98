/*
 * cpu_baseline/ipt_cpu.c -- a tuned parallel CPU implementation of C2R,
 * a STRONGER CPU BASELINE for bench.py only: not a product path (the library has no CPU
 * fallback) and not the oracle (oracle/ stays the plain, untuned checker).
 *
 * Method: Algorithm 1 in gather form, as the paper's CPU version
 * (§5.1): pre-rotation r_j(i) = (i + floor(j/b)) mod m (Eq. 23), row
 * gather d'^{-1}_i(j) (Eq. 31), column gather s'_j(i) = (j + i n -
 * floor(i/a)) mod m (Eq. 26).  Tuning: OpenMP over rows / column panels, column steps on
 * panels of PANEL adjacent columns (whole cache lines per gathered row), one scratch
 * buffer per thread (O(max(m,n)) per worker, Theorem 6).
 */
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef int64_t i64;
#define PANEL 16

static i64 md(i64 x, i64 m) { i64 r = x % m; return r < 0 ? r + m : r; }
static i64 gcd_(i64 x, i64 y) { while (y) { i64 t = x % y; x = y; y = t; } return x; }
static i64 mmi_(i64 a, i64 b) {  /* a^{-1} mod b (extended Euclid), b >= 1 */
    if (b == 1) return 0;
    i64 t = 0, nt = 1, r = b, nr = md(a, b);
    while (nr) { i64 q = r / nr, x = t - q * nt; t = nt; nt = x; x = r - q * nr; r = nr; nr = x; }
    return md(t, b);
}

#define DEFINE_C2R(NAME, T)                                                                    \
static int NAME(T *A, i64 m, i64 n) {                                                          \
    const i64 c = gcd_(m, n), a = m / c, b = n / c, ainv = mmi_(a, b);                         \
    const i64 mx = m > n ? m : n;                                                              \
    int fail = 0;                                                                              \
    _Pragma("omp parallel")                                                                    \
    {                                                                                          \
        T *tmp = (T *)malloc((size_t)(mx * PANEL) * sizeof(T));                                \
        if (!tmp) {                                                                            \
            _Pragma("omp atomic write") fail = 1;                                              \
        }                                                                                      \
        _Pragma("omp barrier")                                                                 \
        if (!fail) {                                                                           \
            if (c > 1) { /* step 1: column pre-rotation, Eq. 23 */                             \
                _Pragma("omp for schedule(dynamic, 4)")                                        \
                for (i64 j0 = 0; j0 < n; j0 += PANEL) {                                        \
                    const i64 w = n - j0 < PANEL ? n - j0 : PANEL;                             \
                    for (i64 jj = 0; jj < w; ++jj) {                                           \
                        const i64 j = j0 + jj, s = (j / b) % m;                                \
                        for (i64 i = 0; i < m; ++i) {                                          \
                            i64 src = i + s; if (src >= m) src -= m;                           \
                            tmp[i * PANEL + jj] = A[src * n + j];                              \
                        }                                                                      \
                    }                                                                          \
                    for (i64 i = 0; i < m; ++i)                                                \
                        for (i64 jj = 0; jj < w; ++jj) A[i * n + j0 + jj] = tmp[i * PANEL + jj]; \
                }                                                                              \
            }                                                                                  \
            /* step 2: row gather, Eq. 31 */                                                   \
            _Pragma("omp for schedule(static)")                                                \
            for (i64 i = 0; i < m; ++i) {                                                      \
                T *row = A + i * n;                                                            \
                memcpy(tmp, row, (size_t)n * sizeof(T));                                       \
                for (i64 j = 0; j < n; ++j) {                                                  \
                    i64 f = j + i * (n - 1);                                                   \
                    if (i - j % c + c > m) f += m;                                             \
                    row[j] = tmp[(ainv * (f / c)) % b + (f % c) * b];                          \
                }                                                                              \
            }                                                                                  \
            /* step 3: column gather, Eq. 26 */                                                \
            _Pragma("omp for schedule(dynamic, 4)")                                            \
            for (i64 j0 = 0; j0 < n; j0 += PANEL) {                                            \
                const i64 w = n - j0 < PANEL ? n - j0 : PANEL;                                 \
                for (i64 i = 0; i < m; ++i) {                                                  \
                    const i64 base = md(i * n - i / a, m);                                     \
                    for (i64 jj = 0; jj < w; ++jj) {                                           \
                        i64 src = base + j0 + jj; src %= m;                                    \
                        tmp[i * PANEL + jj] = A[src * n + j0 + jj];                            \
                    }                                                                          \
                }                                                                              \
                for (i64 i = 0; i < m; ++i)                                                    \
                    for (i64 jj = 0; jj < w; ++jj) A[i * n + j0 + jj] = tmp[i * PANEL + jj];   \
            }                                                                                  \
        }                                                                                      \
        free(tmp);                                                                             \
    }                                                                                          \
    return fail ? -1 : 0;                                                                      \
}

DEFINE_C2R(c2r_u32, uint32_t)
DEFINE_C2R(c2r_u64, uint64_t)

/* C2R(m, n): the row-major m x n buffer becomes its n x m transpose (P_{m,n}).  eb in {4, 8}.
 * Returns 0, -1 on allocation failure, -2 on bad arguments. */
int ipt_cpu_c2r(void *A, i64 m, i64 n, int eb) {
    if (m < 0 || n < 0 || (eb != 4 && eb != 8)) return -2;
    if (m <= 1 || n <= 1) return 0;
    return eb == 4 ? c2r_u32((uint32_t *)A, m, n) : c2r_u64((uint64_t *)A, m, n);
}

int ipt_cpu_threads(void) { return omp_get_max_threads(); }
