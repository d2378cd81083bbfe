/* hostbw.c — host DRAM copy bandwidth (OpenMP, 2 GiB per array), the CPU
 * roofline the oracle's cpu_baseline is reported against (SURVEY.md §8(d):
 * "host DRAM bandwidth is measured in the same run").  Not oracle arithmetic;
 * built and called by bench.py.  Returns GB/s counting read + write bytes. */
#include <stdlib.h>
#include <string.h>
#include <omp.h>

double host_copy_gbs(long long n_doubles, int reps) {
    double *a = malloc(sizeof(double) * n_doubles), *b = malloc(sizeof(double) * n_doubles);
    double best = 0.0;
    long long i;
    int r;
    if (!a || !b) { free(a); free(b); return 0.0; }
#pragma omp parallel for schedule(static)
    for (i = 0; i < n_doubles; i++) { a[i] = (double)i; b[i] = 0.0; }
    for (r = 0; r < reps; r++) {
        double t0 = omp_get_wtime(), t;
#pragma omp parallel for schedule(static)
        for (i = 0; i < n_doubles; i++) b[i] = a[i];
        t = omp_get_wtime() - t0;
        if (t > 0 && 16.0 * n_doubles / t / 1e9 > best) best = 16.0 * n_doubles / t / 1e9;
    }
    free(a); free(b);
    return best;
}
