/* hostbw.c — host DRAM bandwidth (OpenMP, 2 GiB per array), the CPU roofline
 * the oracle's cpu_baseline is reported against ("host DRAM
 * bandwidth is measured in the same run").  Not oracle arithmetic; built and
 * called by bench.py.
 *
 * host_copy_gbs: b[i] = a[i] with ordinary stores, so every written line is
 *   first read into the cache (write-allocate): 24 B of DRAM traffic per
 *   element (read a, read b, write b), which is what is counted.
 * host_read_gbs: a sum reduction over a (8 B per element, read only).
 * The oracle's own algorithmic bytes count no write-allocate and its loops
 * are read-heavy, so bench.py sets them against max(copy, read). */
#include <stdlib.h>
#include <string.h>
#include <omp.h>

/* the OpenMP runtime is shared with the oracle library in bench.py's process
 * (its 1-thread sample calls omp_set_num_threads(1)): set the team size here */
void host_set_threads(int threads) {
    if (threads > 0) omp_set_num_threads(threads);
}

static double* filled(long long n) {
    double* a = malloc(sizeof(double) * n);
    long long i;
    if (!a) return NULL;
#pragma omp parallel for schedule(static)
    for (i = 0; i < n; i++) a[i] = (double)(i & 1023);
    return a;
}

double host_copy_gbs(long long n_doubles, int reps) {
    double *a = filled(n_doubles), *b = filled(n_doubles);
    double best = 0.0;
    long long i;
    int r;
    if (!a || !b) { free(a); free(b); return 0.0; }
    for (r = 0; r < reps; r++) {
        double t0 = omp_get_wtime(), t;
#pragma omp parallel for schedule(static)
        for (i = 0; i < n_doubles; i++) b[i] = a[i];
        t = omp_get_wtime() - t0;
        if (t > 0 && 24.0 * n_doubles / t / 1e9 > best) best = 24.0 * n_doubles / t / 1e9;
    }
    free(a); free(b);
    return best;
}

double host_read_gbs(long long n_doubles, int reps) {
    double* a = filled(n_doubles);
    double best = 0.0, sink = 0.0;
    long long i;
    int r;
    if (!a) return 0.0;
    for (r = 0; r < reps; r++) {
        double t0 = omp_get_wtime(), t, s = 0.0;
#pragma omp parallel for schedule(static) reduction(+ : s)
        for (i = 0; i < n_doubles; i++) s += a[i];
        t = omp_get_wtime() - t0;
        sink += s;
        if (t > 0 && 8.0 * n_doubles / t / 1e9 > best) best = 8.0 * n_doubles / t / 1e9;
    }
    free(a);
    return sink == -1.0 ? 0.0 : best;
}
