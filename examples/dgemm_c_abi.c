/*
 * dgemm_c_abi.c -- using libpdl from C through the C ABI only (include/libpdl.h):
 * load a PDL descriptor, record the paper's DGEMM task on host memory, run it,
 * read the mapping back through the query API, and check a few entries against
 * a direct dot product.  No Python, no torch.
 *
 *   make examples            ->  examples/dgemm_c_abi
 *   examples/dgemm_c_abi [descriptor.xml] [n]
 */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "../include/libpdl.h"

static int check(int rc, const char *what) {
    if (rc < 0) {
        fprintf(stderr, "%s failed (%d): %s\n", what, rc, pdl_last_error());
        exit(1);
    }
    return rc;
}

int main(int argc, char **argv) {
    const char *desc = argc > 1 ? argv[1] : "paper_conf_ipps_sandrieserbp11_b200/descriptors/b200_x1.xml";
    const int64_t n = argc > 2 ? atoll(argv[2]) : 2048;
    double *A = (double *)malloc(sizeof(double) * n * n);
    double *B = (double *)malloc(sizeof(double) * n * n);
    double *C = (double *)malloc(sizeof(double) * n * n);
    if (!A || !B || !C) return 1;
    unsigned s = 12345u;   /* small LCG: values in [0, 1) */
    for (int64_t i = 0; i < n * n; ++i) {
        s = s * 1664525u + 1013904223u;
        A[i] = (s >> 8) * (1.0 / 16777216.0);
        s = s * 1664525u + 1013904223u;
        B[i] = (s >> 8) * (1.0 / 16777216.0);
    }
    char buf[256];
    check(pdl_query("version", buf, sizeof buf), "pdl_query(version)");
    printf("%s\n", buf);
    check(pdl_load(desc), "pdl_load");
    check(pdl_query("workers", buf, sizeof buf), "pdl_query(workers)");
    printf("gpu Workers in the descriptor: %s\n", buf);
    check(task_matmul(A, B, C, n, n, n, 256), "task_matmul");
    check(pdl_run(), "pdl_run");
    /* bytes moved along the descriptor's interconnects: with several Workers joined
       by NVLink, host operands cross PCIe once and the panels move Worker<->Worker */
    char stats[8192];
    check(pdl_query("stats", stats, sizeof stats), "pdl_query(stats)");
    const char *tr = strstr(stats, "\"transfers\"");
    if (tr) {
        const char *end = strchr(tr, '}');
        printf("%.*s}\n", end ? (int)(end - tr) : (int)strlen(tr), tr);
    }
    int64_t plan[PDL_PLAN_LEN];
    check(pdl_plan(n, n, n, 256, NULL, 0, plan, PDL_PLAN_LEN), "pdl_plan");
    printf("Worker 0 of %lld: rows [%lld, %lld) cols [%lld, %lld), %lld x %lld tile tasks in all\n",
           (long long)plan[0], (long long)plan[5], (long long)plan[6], (long long)plan[7], (long long)plan[8],
           (long long)plan[11], (long long)plan[12]);
    double worst = 0.0;
    for (int t = 0; t < 64; ++t) {   /* sampled entries against a direct dot product */
        const int64_t i = (t * 7919) % n, j = (t * 104729) % n;
        double ref = 0.0, den = 0.0;
        for (int64_t k = 0; k < n; ++k) {
            ref += A[i * n + k] * B[k * n + j];
            den += fabs(A[i * n + k]) * fabs(B[k * n + j]);
        }
        const double e = fabs(C[i * n + j] - ref) / den;
        if (e > worst) worst = e;
    }
    printf("max scaled error on 64 sampled entries: %.3e\n", worst);
    pdl_unload();
    free(A);
    free(B);
    free(C);
    return worst <= 1e-12 ? 0 : 2;
}
