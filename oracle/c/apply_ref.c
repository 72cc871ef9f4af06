/* ORACLE — test infrastructure only (bench.py cpu_baseline / --impl reference).
 *
 * The offline permutation by its definition, PAPER.md L361 / L365
 * (D-designated algorithm): for i in 0..n-1: b[p[i]] = a[i].
 * A plain loop over raw words; OpenMP splits the index range over the host
 * cores (the loop body is untouched). No blocking, no reordering.
 */
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

void oracle_apply_u32(const int32_t* p, const uint32_t* a, uint32_t* b, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) b[p[i]] = a[i];
}

void oracle_apply_u64(const int32_t* p, const uint64_t* a, uint64_t* b, int64_t n) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) b[p[i]] = a[i];
}

int oracle_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
