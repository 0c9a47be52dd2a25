/*
 * su3.c -- oracle for the SU3Bench mat_nn kernel (config 3).
 * TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * The paper's SU3Bench is "a sparse matrix-matrix multiply routine for the
 * Special Unitary group of order 3" extracted from MILC, run as
 * version 0, the CPU-style OpenMP code.  For each
 * lattice site s and link direction j the kernel forms the 3x3 complex product
 * C[s][j] = A[s][j] * B[j].  This is the plain definition:
 * accumulator starts at 0+0i, m runs 0,1,2, each complex multiply-add is
 *   re += ar*br - ai*bi ;  im += ar*bi + ai*br
 * with every product rounded before the subtraction/addition (no FMA).
 * fp64 per BASELINE.json config 3 (the paper timed f32; AMB-8).
 */
#include "oracle.h"
#include <pthread.h>
#include <stdlib.h>

typedef struct {
    int64_t lo, hi;
    const double *A, *B;
    double *C;
} su3_job;

static void *su3_worker(void *p)
{
    su3_job *jb = p;
    for (int64_t s = jb->lo; s < jb->hi; s++)
        for (int j = 0; j < 4; j++)
            for (int k = 0; k < 3; k++)
                for (int l = 0; l < 3; l++) {
                    double re = 0.0, im = 0.0;
                    for (int m = 0; m < 3; m++) {
                        const double *a = &jb->A[((((s * 4 + j) * 3 + k) * 3) + m) * 2];
                        const double *b = &jb->B[(((j * 3 + m) * 3) + l) * 2];
                        double rr = a[0] * b[0];
                        double ii = a[1] * b[1];
                        double ri = a[0] * b[1];
                        double ir = a[1] * b[0];
                        re += rr - ii;
                        im += ri + ir;
                    }
                    double *c = &jb->C[((((s * 4 + j) * 3 + k) * 3) + l) * 2];
                    c[0] = re;
                    c[1] = im;
                }
    return NULL;
}

void orc_su3_mat_nn(int64_t sites, const double *A, const double *B, double *C, int nthreads)
{
    if (nthreads < 1) nthreads = 1;
    su3_job *jobs = calloc((size_t)nthreads, sizeof(su3_job));
    pthread_t *th = calloc((size_t)nthreads, sizeof(pthread_t));
    for (int w = 0; w < nthreads; w++) {
        jobs[w].lo = sites * w / nthreads;
        jobs[w].hi = sites * (w + 1) / nthreads;
        jobs[w].A = A; jobs[w].B = B; jobs[w].C = C;
    }
    if (nthreads == 1)
        su3_worker(&jobs[0]);
    else {
        for (int w = 0; w < nthreads; w++) pthread_create(&th[w], NULL, su3_worker, &jobs[w]);
        for (int w = 0; w < nthreads; w++) pthread_join(th[w], NULL);
    }
    free(jobs);
    free(th);
}
