/* Host microbenchmark of the selector (kernel selection must not add
 * visible time).  For every shape of the bench workloads: the first adaptic_plan call (fills
 * the selector's memo cell) and the mean of N further adaptic_plan + adaptic_plan_destroy
 * pairs, in ns, with clock_gettime(CLOCK_MONOTONIC).  Prints one JSON object.
 *   gcc -O2 -Iinclude tools/plan_latency.c -Lpaper_conf_pldi_samadihmlm12_b200 -ladaptic \
 *       -Wl,-rpath,'$ORIGIN/../paper_conf_pldi_samadihmlm12_b200' -o tools/plan_latency        */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <time.h>
#include "adaptic.h"

static double now_ns(void) {
    struct timespec t;
    clock_gettime(CLOCK_MONOTONIC, &t);
    return t.tv_sec * 1e9 + t.tv_nsec;
}
static int cmp(const void* a, const void* b) {
    double x = *(const double*)a, y = *(const double*)b;
    return (x > y) - (x < y);
}

int main(int argc, char** argv) {
    const int iters = argc > 1 ? atoi(argv[1]) : 2000;
    int64_t shapes[128][3];
    int n = 0;
    for (int k = 3; k <= 23; ++k)
        for (int op = 0; op < 2; ++op) {
            shapes[n][0] = op; shapes[n][1] = (int64_t)1 << k; shapes[n][2] = (int64_t)1 << (26 - k); ++n;
            shapes[n][0] = op; shapes[n][1] = ((int64_t)1 << k) + (op == 1); shapes[n][2] = ((int64_t)1 << (26 - k)) + (op == 0); ++n;
        }
    shapes[n][0] = 1; shapes[n][1] = 256; shapes[n][2] = 256; ++n;                       /* configs[0] */
    for (int k = 10; k <= 30; k += 4) { shapes[n][0] = 2; shapes[n][1] = 1; shapes[n][2] = (int64_t)1 << k; ++n; }
    shapes[n][0] = 0; shapes[n][1] = 131072; shapes[n][2] = 32768; ++n;                  /* configs[3] */
    shapes[n][0] = 1; shapes[n][1] = 1024; shapes[n][2] = (int64_t)1 << 24; ++n;          /* configs[4] */
    double warm[128], cold[128];
    {   /* the first call on a GPU box creates the CUDA context (~0.3 s): not selector time */
        adaptic_plan_t p0;
        if (adaptic_plan(ADAPTIC_OP_STENCIL5, 3, 3, ADAPTIC_F32, &p0) == ADAPTIC_OK) adaptic_plan_destroy(p0);
    }
    for (int i = 0; i < n; ++i) {
        adaptic_plan_t p;
        double t0 = now_ns();
        if (adaptic_plan((adaptic_op)shapes[i][0], shapes[i][1], shapes[i][2], ADAPTIC_F32, &p) != ADAPTIC_OK) return 1;
        cold[i] = now_ns() - t0;
        adaptic_plan_destroy(p);
        t0 = now_ns();
        for (int j = 0; j < iters; ++j) {
            adaptic_plan((adaptic_op)shapes[i][0], shapes[i][1], shapes[i][2], ADAPTIC_F32, &p);
            adaptic_plan_destroy(p);
        }
        warm[i] = (now_ns() - t0) / iters;
    }
    if (getenv("PLAN_VERBOSE")) for (int i = 0; i < n; ++i) fprintf(stderr, "%lld %lld %lld %.0f\n", (long long)shapes[i][0], (long long)shapes[i][1], (long long)shapes[i][2], warm[i]);
    double ws[128], cs[128];
    for (int i = 0; i < n; ++i) { ws[i] = warm[i]; cs[i] = cold[i]; }
    qsort(ws, n, sizeof(double), cmp);
    qsort(cs, n, sizeof(double), cmp);
    int worst = 0;
    for (int i = 1; i < n; ++i) if (warm[i] > warm[worst]) worst = i;
    printf("{\"shapes\": %d, \"iters\": %d, \"plan_ns_median\": %.1f, \"plan_ns_p90\": %.1f, \"plan_ns_max\": %.1f, "
           "\"worst\": [%lld, %lld, %lld], \"first_call_ns_median\": %.1f, \"first_call_ns_max\": %.1f}\n",
           n, iters, ws[n / 2], ws[(int)(0.9 * (n - 1))], ws[n - 1], (long long)shapes[worst][0],
           (long long)shapes[worst][1], (long long)shapes[worst][2], cs[n / 2], cs[n - 1]);
    return 0;
}
