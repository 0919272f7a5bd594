/* cpu_csr_omp.c -- NOT the oracle: a multi-threaded fp64 CSR SpMV used only
 * as context for bench.py's CPU baseline ("an OpenMP
 * row-parallel CSR SpMV on all cores available to the process").  Test and
 * measurement infrastructure like the rest of oracle/; the product path
 * never loads it.  Plain definition of y = A x (Alg. 1) with one
 * fp64 running sum per row, rows split statically over the threads. */
#include <stdint.h>
#include <omp.h>

int cpu_csr_omp_threads(void) { return omp_get_max_threads(); }

void cpu_csr_omp_spmv(int64_t m, const int32_t *rowptr, const int32_t *colidx, const double *val,
                      const double *x, double *y) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        double s = 0.0;
        for (int32_t k = rowptr[i]; k < rowptr[i + 1]; ++k) s += val[k] * x[colidx[k]];
        y[i] = s;
    }
}
