/*
 * oracle.h -- plain, slow, obviously-correct CPU oracle for the OpenMP device-runtime hot
 * path of Doerfert et al., "Co-Designing an OpenMP GPU Runtime and Optimizations for
 * Near-Zero Overhead Execution" (IPDPS'22).  Citations "P:<line> §<sec>" point into
 * /root/reference/PAPER.md; "SURVEY §x" into /root/repo/SURVEY.md (the readings of the
 * paper adopted by this build, listed again in DESIGN.md).
 *
 * THIS IS TEST INFRASTRUCTURE.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg may load it.  It shares no code, header, table or
 * constant generator with the CUDA path (paper_conf_ipps_doerfertphtdcg22_b200/csrc) and
 * neither side includes the other.  Built with `gcc -O2 -ffp-contract=off` so that every
 * a*b+c below rounds twice unless written as fma().
 *
 * Parity status per function:
 *   schedule (closed form + literal Fig. 5)  pinned: brute force vs each other, exactly-once
 *   axpy / sums                              pinned: integer-valued closed form 2^30, long-double
 *   generic-mode semantics + ICVs            pinned: brute-force per-thread emulation, closed forms
 *   XSBench-shaped lookup                    pinned: textbook upper_bound, nuclide-grid search,
 *                                            LCG brute force, endpoint interpolation;
 *                                            XSBench published checksum: "parity unpinned"
 *   RSBench-shaped lookup                    pinned: Faddeeva vs scipy wofz / erfc, fast_exp closed
 *                                            form, window bracketing; whole-lookup value
 *                                            "partially pinned" (no published value)
 *   SU(3)                                    pinned: B=I, A=1,B=1/3 closed forms, numpy einsum
 */
#ifndef OMPRT_ORACLE_H
#define OMPRT_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- Fig. 5 static schedule (§III-F) ---------------------------------------- */
/* Closed form of the combined distribute-parallel-for schedule without chunks:
 * iteration iv runs on global thread g = iv mod (T*N): team g/N, thread g%N.
 * Returns 0, or -1 when iv is outside [0,n) (nothing runs it). */
int oracle_static_owner_closed(int64_t iv, int64_t n, int64_t teams, int64_t threads,
                               int32_t *team, int32_t *thread);
/* Literal transliteration of Fig. 5's noChunkImpl, simulated for every (BId, TId) in order.
 * owner[iv] = BId*NumThreads+TId (global thread id), count[iv] = times iv ran.
 * With assume_oversub the loop breaks after one iteration. */
void oracle_fig5_simulate(int64_t n, int32_t teams, int32_t threads, int assume_oversub,
                          int32_t *owner, int32_t *count);
/* Q2 reading: `for` within one team = Fig. 5 with NumBlocks=1, BId=0; `distribute` alone
 * = Fig. 5 with NumThreads=1, TId=0.  owner = thread (resp. team) that runs iv. */
void oracle_team_for_simulate(int64_t n, int32_t nthreads, int assume_oversub,
                              int32_t *owner, int32_t *count);
void oracle_distribute_simulate(int64_t n, int32_t teams, int32_t *owner, int32_t *count);

/* NEXT f3 (Fig. 5 covers only "the absence of user-defined chunks"; reading R-F3):
 * static schedule with a user chunk C applied to the combined scheme, OpenMP round-robin:
 * chunk k = iterations [kC, min(n, kC + C)) runs on global thread k mod (T*N).  C = 1 is
 * Fig. 5.  Closed form and a literal per-thread simulation. */
int oracle_static_chunk_owner_closed(int64_t iv, int64_t n, int64_t chunk, int64_t teams,
                                     int64_t threads, int32_t *team, int32_t *thread);
void oracle_chunk_simulate(int64_t n, int64_t chunk, int32_t teams, int32_t threads,
                           int assume_oversub, int32_t *owner, int32_t *count);
/* Reading R-D1: schedule(dynamic, C) under a blocked distribute (team of iteration iv, and
 * a literal execution for one seeded request order). */
int oracle_dynamic_team_closed(int64_t iv, int64_t n, int64_t teams);
void oracle_dynamic_simulate(int64_t n, int64_t chunk, int32_t teams, int32_t threads,
                             uint64_t order_seed, int32_t *owner, int32_t *count);

/* ---- C1: SPMD axpy + fp64 sum reduction (BASELINE configs[0]) -------------------------- */
/* a[i] = fma(x, b[i], c[i]) (SURVEY Q12 reading: one rounding, explicit). */
void oracle_axpy(int64_t n, double x, const double *b, const double *c, double *a);
/* OpenMP reduction(+): init + sum v[i], computed with Neumaier compensation in double. */
double oracle_sum_f64(const double *v, int64_t n, double init);
/* Same in long double (x87 80-bit) with Neumaier compensation: a second, independent
 * high-accuracy reference used to pin the first. */
long double oracle_sum_f64_ld(const double *v, int64_t n, double init);
/* sum |v[i]| (for the relative tolerance bound). */
double oracle_sum_abs_f64(const double *v, int64_t n);

/* ---- reductions (north_star; the paper did not redesign them) --------------------- */
enum { ORACLE_OP_ADD = 0, ORACLE_OP_MUL = 1, ORACLE_OP_MIN = 2, ORACLE_OP_MAX = 3 };
/* orig (+) (op over v) for u64 (wrapping mod 2^64). */
uint64_t oracle_reduce_u64(const uint64_t *v, int64_t n, int op, uint64_t orig);
/* orig (op) (op over v) for f64; ADD uses Neumaier, MUL/MIN/MAX sequential. */
double oracle_reduce_f64(const double *v, int64_t n, int op, double orig);

/* ---- C2: generic-mode team kernel (§II-C, §III-D) -------- */
/* For each team t sequentially: the main thread runs the prologue over "globalized"
 * team arrays w[inner_n], perm[inner_n] (alloc_shared), then a parallel region of
 * nthreads threads runs the team `for` j -> thread j mod nthreads:
 *   out[t*inner_n+j] = w[perm[j]] / s + w[j],   owner[t*inner_n+j] = thread number.
 * postlogue[t] (nullable) = sequential sum of out[t*inner_n + 0..inner_n) after the join. */
void oracle_generic_team(int32_t teams, int32_t nthreads, int32_t inner_n, const double *in,
                         double *out, int32_t *owner, double *postlogue);

/* ICV queries (§III-B..E; values per OpenMP 5.1).
 * Record layout per query point: 7 int32 = thread_num, num_threads, level, active_level,
 * in_parallel, team_num, num_teams.  For team t the output holds
 *   [prologue (main only)] [region thread 0..nthreads-1] [nested region thread 0..]
 *   [after nested, thread 0..]
 * i.e. (1 + 3*nthreads) records per team.  Nested parallel regions are serialized
 * (P:116-117): they get one thread. */
#define ORACLE_ICV_FIELDS 7
void oracle_icv_table(int32_t teams, int32_t nthreads, int32_t nested_request, int32_t *rec);

/* ---- C3: XSBench-shaped macroscopic cross-section lookup (§V-A) --- */
uint64_t oracle_lcg_fast_forward(uint64_t seed, uint64_t n);
uint64_t oracle_lcg_step(uint64_t seed, uint64_t n);          /* n sequential steps (brute force) */
double oracle_lcg_double(uint64_t *seed);
int oracle_pick_mat(uint64_t *seed);
int64_t oracle_grid_search(const double *A, int64_t len, double quarry);
typedef struct {
  int32_t n_isotopes, n_gridpoints, max_num_nucs, pad;
  int64_t n_union;
  const double *nuclide_grid;  /* [n_isotopes*n_gridpoints][6] */
  const double *unionized;     /* [n_union] */
  const int32_t *index_grid;   /* [n_union][n_isotopes] */
  const int32_t *num_nucs;     /* [12] */
  const int32_t *mats;         /* [12][max_num_nucs] */
  const double *concs;         /* [12][max_num_nucs] */
} oracle_xs_tables;
/* Lookups [first, first+count): verification[i-first] = 1 + argmax of the 5 macro xs.
 * macro (nullable): [count][5].  Returns 0. */
int oracle_xs_lookup(const oracle_xs_tables *t, uint64_t seed, int64_t first, int64_t count,
                     uint64_t *verification, double *macro);
/* Same lookups via a per-nuclide binary search of the energy instead of the unionized
 * index grid (XSBench's "nuclide grid" method): an independent pin of the index grid. */
int oracle_xs_lookup_nuclide_search(const oracle_xs_tables *t, uint64_t seed, int64_t first,
                                    int64_t count, uint64_t *verification, double *macro);
/* Algorithmic bytes of lookups [first, first+count) (table elements read + the verification
 * store), for the roofline's per-unit figure. */
int64_t oracle_xs_bytes(const oracle_xs_tables *t, uint64_t seed, int64_t first, int64_t count);

/* ---- C4: RSBench-shaped multipole lookup (§V-A) ------------------ */
double oracle_fast_exp(double x);
void oracle_fast_nuclear_W(double zr, double zi, double *wr, double *wi);
typedef struct {
  int32_t n_nuclides, numL, max_num_nucs, pad;
  const double *poles;       /* [n_poles][8] EA RT RA RF (re,im) */
  const int32_t *pole_l;     /* [n_poles] */
  const double *windows;     /* [n_windows][4] T A F 0 */
  const int32_t *win_range;  /* [n_windows][2] absolute pole [start,end) */
  const int32_t *win_off;    /* [n_nuclides+1] */
  const int32_t *n_windows;  /* [n_nuclides] */
  const double *k0rs;        /* [n_nuclides][numL] */
  const int32_t *num_nucs;
  const int32_t *mats;
  const double *concs;
} oracle_rs_tables;
/* verification[i-first] = 1 + argmax of 4 macro xs; macro (nullable) [count][4]. */
int oracle_rs_lookup(const oracle_rs_tables *t, uint64_t seed, int64_t first, int64_t count,
                     uint64_t *verification, double *macro);
/* Instrumented pass over lookups [first,first+count) (the C4 roofline's per-unit figure,
 * SURVEY §8(d)): ops[10] = {add/sub, mul, div, sqrt, transcendental calls, Faddeeva
 * evaluations, of them Abrarov, poles visited, (lookup, nuclide) pairs, fma}. */
void oracle_rs_count(const oracle_rs_tables *t, uint64_t seed, int64_t first, int64_t count,
                     int64_t *ops);

/* ---- C5: SU(3) link multiply (GridMini-shaped) --------------- */
/* C[s][l] = A[s][l] x B[l] (3x3 complex), complex MAC as 4 explicit fmas in fixed order. */
void oracle_su3_mult(const double *A, const double *B, double *C, int64_t n_sites);

#ifdef __cplusplus
}
#endif
#endif
