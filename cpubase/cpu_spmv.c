/*
 * cpu_spmv.c -- a realistic CPU SpMV baseline, NOT the oracle:
 * y = alpha*A*x + beta*y over CSR rows [0, m), fp64 accumulation, OpenMP over rows on all
 * host cores (dynamic chunks for skewed rows), compiled -O3 (portable x86-64).  bench.py
 * reports it beside the oracle (long double, as written) so the GPU/CPU ratio has a
 * sensible CPU denominator as well as the deliberately slow checker.
 */
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

void cpu_spmv_f64(int64_t m, const int64_t *row_ptr, const int32_t *col, const double *val, const double *x,
                  double alpha, double beta, double *y)
{
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t r = 0; r < m; ++r) {
        double s = 0.0;
        for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k) s += val[k] * x[col[k]];
        y[r] = beta != 0.0 ? alpha * s + beta * y[r] : alpha * s;
    }
}

int cpu_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
