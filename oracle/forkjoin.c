/*
 * forkjoin.c -- oracle for the fork/join microbenchmark (config 2) and a real
 * host thread team that executes the same program (the CPU baseline).
 * TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * Program of one team g (SURVEY.md 8(a) a2-a7, 8(a') "Fork/join bench";
 * PAPER P:606-625 generic mode: the main thread runs the sequential code and
 * hands each parallel region to the workers, who run it and go back to
 * waiting):
 *
 *   for r in 0..R-1:                         # sequential region (main)
 *       v_r = g*R + r                        # body 2 only: produced by main
 *       parallel region k_r = r mod K         # fork ... join
 *           worker t (0..T-1):  body 1: acc_t += (k_r+1)*(r+1)*(t+1)
 *                               body 2: acc_t += v_r
 *       body 0: count += 1                   # main, after the join
 *   result = count (body 0)  or  sum_t acc_t (bodies 1, 2)
 */
#include "oracle.h"
#include <pthread.h>
#include <stdlib.h>
#include <time.h>

uint64_t orc_fj_team(int32_t g, int32_t T, int64_t R, int32_t body, int32_t K)
{
    uint64_t count = 0;
    uint64_t *acc = calloc((size_t)T, sizeof(uint64_t));
    for (int64_t r = 0; r < R; r++) {
        uint64_t v = (uint64_t)g * (uint64_t)R + (uint64_t)r;
        uint64_t k = (uint64_t)(r % K);
        for (int32_t t = 0; t < T; t++) {          /* the region, per worker */
            if (body == 1)
                acc[t] += (k + 1) * (uint64_t)(r + 1) * (uint64_t)(t + 1);
            else if (body == 2)
                acc[t] += v;
        }
        if (body == 0)
            count += 1;
    }
    uint64_t res = count;
    if (body != 0)
        for (int32_t t = 0; t < T; t++)
            res += acc[t];
    free(acc);
    return res;
}

/* ---- a real host team: 1 main thread + T workers, pthread barriers ---- */
typedef struct {
    pthread_barrier_t fork_bar, join_bar;
    volatile int64_t r;        /* work descriptor: region index, -1 = terminate */
    volatile uint64_t v;
    int32_t body, K, T;
    uint64_t *acc;
} host_team;

typedef struct { host_team *tm; int32_t t; } host_worker;

static void *worker_loop(void *p)
{
    host_worker *w = p;
    host_team *tm = w->tm;
    for (;;) {
        pthread_barrier_wait(&tm->fork_bar);
        int64_t r = tm->r;
        if (r < 0)
            break;
        uint64_t k = (uint64_t)(r % tm->K);
        if (tm->body == 1)
            tm->acc[w->t] += (k + 1) * (uint64_t)(r + 1) * (uint64_t)(w->t + 1);
        else if (tm->body == 2)
            tm->acc[w->t] += tm->v;
        pthread_barrier_wait(&tm->join_bar);
    }
    return NULL;
}

uint64_t orc_fj_host_team(int32_t T, int64_t R, int32_t body, int32_t K, double *ns)
{
    host_team tm;
    tm.body = body; tm.K = K; tm.T = T;
    tm.acc = calloc((size_t)T, sizeof(uint64_t));
    pthread_barrier_init(&tm.fork_bar, NULL, (unsigned)T + 1);
    pthread_barrier_init(&tm.join_bar, NULL, (unsigned)T + 1);
    pthread_t *th = calloc((size_t)T, sizeof(pthread_t));
    host_worker *ws = calloc((size_t)T, sizeof(host_worker));
    for (int32_t t = 0; t < T; t++) {
        ws[t].tm = &tm;
        ws[t].t = t;
        pthread_create(&th[t], NULL, worker_loop, &ws[t]);
    }
    struct timespec a, b;
    clock_gettime(CLOCK_MONOTONIC, &a);
    uint64_t count = 0;
    for (int64_t r = 0; r < R; r++) {
        tm.v = (uint64_t)r;                       /* g = 0 for the host team */
        tm.r = r;
        pthread_barrier_wait(&tm.fork_bar);       /* fork */
        pthread_barrier_wait(&tm.join_bar);       /* join */
        if (body == 0)
            count += 1;
    }
    clock_gettime(CLOCK_MONOTONIC, &b);
    tm.r = -1;
    pthread_barrier_wait(&tm.fork_bar);           /* terminate */
    for (int32_t t = 0; t < T; t++)
        pthread_join(th[t], NULL);
    if (ns)
        *ns = ((double)(b.tv_sec - a.tv_sec) * 1e9 + (double)(b.tv_nsec - a.tv_nsec)) / (double)R;
    uint64_t res = count;
    if (body != 0)
        for (int32_t t = 0; t < T; t++)
            res += tm.acc[t];
    pthread_barrier_destroy(&tm.fork_bar);
    pthread_barrier_destroy(&tm.join_bar);
    free(tm.acc);
    free(th);
    free(ws);
    return res;
}
