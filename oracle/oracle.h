/*
 * oracle.h -- plain, slow, single-threaded-by-definition CPU oracle for the
 * hot path of Huber et al., "Efficient Execution of OpenMP on GPUs" (CGO'22).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load liboracle.so.
 * The product path (libgtr.so + its Python binding) never links, loads or
 * calls anything here, and this code shares nothing with it: no headers, no
 * helpers, no constants, no table builders.  The only code both sides use is
 * the seeded input generator package gtr_inputs/ (table contents only).
 *
 * Compiled with -O2 -ffp-contract=off -fno-fast-math: IEEE binary64,
 * round-to-nearest-even, every multiply and add rounded separately.
 * Unsigned 64-bit wrap-around arithmetic for the LCG.
 *
 * Citation format: P:a-b = /root/reference/PAPER.md lines a-b.  Where the
 * paper is silent the reading is SURVEY.md 8(c) / DESIGN.md "Readings".
 *
 * Pin status: every function below is pinned by a
 * `-m "not gpu"` test except where marked "parity unpinned".
 */
#ifndef GTR_ORACLE_H
#define GTR_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------- lookup sampling (paper silent) -------- */
uint64_t orc_lcg_next(uint64_t s);                 /* (a*s + c) mod 2^63 */
double   orc_lcg_double(uint64_t *seed);           /* advance, return s/2^63 */
uint64_t orc_lcg_ff(uint64_t seed, uint64_t n);    /* n steps in O(log n) */
int      orc_pick_mat(uint64_t *seed);             /* XSBench material draw */

/* ---------------- XSBench unionized-grid lookup (config 1, 5) ----------- */
typedef struct {
    int64_t n_iso, n_gp, n_union;
    int32_t max_num_nucs;
    const double  *grid;        /* [n_iso][n_gp][6] sorted per nuclide      */
    const double  *egrid;       /* [n_union] unionized energies, ascending  */
    const int32_t *index_grid;  /* [n_union][n_iso]                         */
    const int32_t *num_nucs;    /* [12]                                     */
    const int32_t *mats;        /* [12][max_num_nucs]                       */
    const double  *concs;       /* [12][max_num_nucs]                       */
    int32_t grid_type;          /* 0 unionized, 1 nuclide, 2 hash (XSBench) */
    int32_t hash_bins;          /* hash grid: number of energy bins         */
    const int32_t *hash_index;  /* [hash_bins][n_iso] (grid_type 2)         */
} orc_xs_tables;

/* egrid = all n_iso*n_gp energies sorted ascending (qsort). */
void    orc_xs_build_egrid(const double *grid, int64_t n_iso, int64_t n_gp, double *egrid);
/* XSBench sequential index rule. */
void    orc_xs_build_index_grid(const double *grid, int64_t n_iso, int64_t n_gp,
                                const double *egrid, int64_t n_union, int32_t *index_grid);
/* lower-bound binary search of XSBench. */
int64_t orc_grid_search(int64_t n, const double *a, double quarry);
/* XSBench's per-nuclide lower-bound search in [low, high] on gridpoint
 * energies (stride 6 doubles). */
int64_t orc_nuclide_search(const double *grid_n, double quarry, int64_t low, int64_t high);
/* Hash grid (XSBench): bin b starts at energy b/hash_bins; hash_index[b][n]
 * = lower-bound index of that energy in nuclide n's grid. */
void    orc_xs_build_hash_grid(const double *grid, int64_t n_iso, int64_t n_gp, int32_t hash_bins,
                               int32_t *hash_index);
/* one lookup, global index i (grid_type selects how the
 * bracketing gridpoint of each nuclide is found: unionized index grid,
 * per-nuclide search, or hash bin + bounded search -- all the same interval). */
void    orc_xs_lookup(const orc_xs_tables *t, uint64_t i, uint64_t seed,
                      int32_t *mat, int64_t *u, double macro[5], int32_t *argmax);
/* lookups [first, first+n): out[0] = hash = sum(argmax+1), out[1..12] material
 * tallies, out[13..17] argmax tallies (ADDED to out).  Optional per-lookup
 * dumps (may be NULL): v_mat u8[n], v_u u32[n], v_am u8[n], v_macro f64[n][5].
 * nthreads > 1 splits the range across pthreads (integer sums: identical). */
void    orc_xs_run(const orc_xs_tables *t, uint64_t first, uint64_t n, uint64_t seed,
                   int nthreads, uint64_t out[18], uint8_t *v_mat, uint32_t *v_u,
                   uint8_t *v_am, double *v_macro);

/* ---------------- SU3Bench mat_nn (config 3) ---------------------------- */
/* C[s][j][k][l] = sum_m A[s][j][k][m] * B[j][m][l]; complex as (re,im). */
void    orc_su3_mat_nn(int64_t sites, const double *A, const double *B, double *C,
                       int nthreads);

/* ---------------- RSBench multipole lookup (config 4) ------------------- */
typedef struct {
    int64_t n_nuc, max_poles, max_windows;
    int32_t max_num_nucs;
    const int32_t *n_windows;   /* [n_nuc] */
    const double  *poles;       /* [n_nuc][max_poles] records of 9 x 8 B:
                                   EA.re EA.im RT.re RT.im RA.re RA.im RF.re RF.im
                                   (l_value:int32, pad:int32)                  */
    const double  *windows;     /* [n_nuc][max_windows] records of 4 x 8 B:
                                   T A F (start:int32, end:int32)              */
    const double  *k0rs;        /* [n_nuc][4] */
    const int32_t *num_nucs, *mats;
    const double  *concs;
} orc_rs_tables;

typedef struct { double r, i; } orc_cplx;
orc_cplx orc_fast_nuclear_W(orc_cplx z);          /* Abrarov / asymptotic   */
/* the tabulated Faddeeva constants orc_fast_nuclear_W uses (for their pins) */
void orc_rs_faddeeva_constants(double an[10], double dl[10], double *prefactor, double asym[4]);
double   orc_fast_exp(double x);                   /* (1+x/4096)^(2^12)      */
void     orc_rs_lookup(const orc_rs_tables *t, uint64_t i, uint64_t seed,
                       int32_t *mat, double macro[4], int32_t *argmax);
void     orc_rs_run(const orc_rs_tables *t, uint64_t first, uint64_t n, uint64_t seed,
                    int nthreads, uint64_t out[18], uint8_t *v_mat, uint8_t *v_am,
                    double *v_macro, double *min_margin);
/* algorithmic fp64 work (see rs.c): counts[0] nuclide visits, [1] Abrarov
 * poles, [2] asymptotic poles (ADDED to counts); flops from the counts,
 * *transcendentals = sin/cos/atan calls.                                   */
#define ORC_RS_FLOPS_NUC  36.0
#define ORC_RS_FLOPS_POLE 35.0
#define ORC_RS_FLOPS_WA   367.0
#define ORC_RS_FLOPS_WB   50.0
void     orc_rs_work(const orc_rs_tables *t, uint64_t first, uint64_t n, uint64_t seed, int nthreads,
                     uint64_t counts[3]);
double   orc_rs_flops(const uint64_t counts[3], double *transcendentals);

/* ---------------- fork/join + runtime semantics (config 2; 8(c) c6) ---- */
/* Per-team results of the fork/join program with T workers and R regions.
 * body: 0 = empty (main counts joins), 1 = trivial (worker t in region r adds
 * (k_r+1)*(r+1)*(t+1), k_r = r mod K), 2 = broadcast (main produces
 * v_r = g*R + r, every worker adds v_r).  Sequential simulation.          */
uint64_t orc_fj_team(int32_t g, int32_t T, int64_t R, int32_t body, int32_t K);
/* Same program executed by a real host thread team (1 main + T-1 workers,
 * pthread barriers for fork and join).  Returns the team result; *ns gets
 * wall ns per fork/join.  CPU baseline for config 2.                      */
uint64_t orc_fj_host_team(int32_t T, int64_t R, int32_t body, int32_t K, double *ns);

/* Expected outputs of the runtime semantic programs (Figs. 1, 3, 5, 7 and
 * nested parallelism), written into out[] per team; see oracle/semantics.c. */
int      orc_sem_expected(int32_t test_id, int32_t num_teams, int32_t T, uint64_t *out,
                          int64_t out_len);

#ifdef __cplusplus
}
#endif
#endif
