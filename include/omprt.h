/*
 * omprt.h -- C ABI of libomprt.so, the B200-native (sm_100a) device-runtime hot path of
 * Doerfert et al., "Co-Designing an OpenMP GPU Runtime and Optimizations for Near-Zero
 * Overhead Execution" (IPDPS'22).  "P:<line> §<sec>" cites /root/reference/PAPER.md.
 *
 * Each entry point launches the execution of one offloaded
 *     #pragma omp target teams distribute parallel for        (SPMD mode)
 * or one generic-mode target region (sequential main thread + `parallel`),
 * driven by the header-only device runtime (csrc/omprt/device: init/deinit P:100-112,
 * Fig. 5 static schedule P:121-149, state machine P:92, alloc_shared stack P:110-112,
 * team/league reductions), and -- under the `omprt_cuda_*` names -- the hand-written bare
 * CUDA kernel of the same loop (the paper's "CUDA (NVCC)" rows), which gives the
 * "overhead versus CUDA".
 *
 * Conventions (all functions):
 *   - Return an int status: OMPRT_OK (0) or a negative OMPRT_E_* code; no C++ exception
 *     crosses the ABI.  omprt_last_error() returns the calling thread's last message.
 *   - Data pointers are DEVICE pointers owned by the caller (e.g. torch tensors) unless the
 *     name says `_host`.  The library never frees caller memory.  It owns only its
 *     per-device workspace (fallback pool, league partials, tickets, error word), created
 *     by omprt_init and released by omprt_fini.
 *   - The device is the calling thread's current CUDA device; omprt_init must have been
 *     called for it (else OMPRT_E_NOTINIT).
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Launches
 *     are asynchronous; results are valid after the stream is synchronized.  Calls that
 *     reduce share the device's league workspace: launch them on one stream (in order).
 *   - Reductions follow OpenMP: *inout = *inout (+) sum over all iterations.
 *   - Device-side fatal errors (stack pool exhausted, debug assertion) record a code in a
 *     mapped host word and trap; omprt_device_status() reports it.
 */
#ifndef OMPRT_H
#define OMPRT_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ------------------------------------------------------------------ */
#define OMPRT_OK 0
#define OMPRT_E_INVAL (-1)   /* bad argument (incl. a violated oversubscription assumption) */
#define OMPRT_E_CUDA (-2)    /* a CUDA runtime call failed (message in omprt_last_error) */
#define OMPRT_E_NOMEM (-3)   /* device allocation failed */
#define OMPRT_E_STACK (-4)   /* shared-memory stack and its global pool exhausted */
#define OMPRT_E_ASSERT (-5)  /* debug-build device assertion failed */
#define OMPRT_E_NOTINIT (-6) /* omprt_init was not called for the current device */

/* ---- launch flags ------------------------------------------------------------------ */
/* P:125 §III-F user assumption: n <= teams*threads (distribute parallel for) or n <= team
 * size (team `for`): every thread runs at most one iteration and the loop disappears.  The
 * host rejects a call that violates it (OMPRT_E_INVAL) instead of dropping iterations. */
#define OMPRT_ASSUME_OVERSUB (1u << 0)
/* Test build: record owner[i] = global thread id that ran iteration i (and count[i]). */
#define OMPRT_RECORD_OWNER (1u << 1)
/* Generic mode: use the general state machine (function pointer) instead of the custom
 * compile-time one. */
#define OMPRT_GENERAL_SM (1u << 2)
/* Generic mode stack placement: dynamic shared memory of 2 KiB / 0 B instead of
 * the static 4 KiB stack, so globalized arrays fall back to the global pool. */
#define OMPRT_SMALL_STACK (1u << 3)
#define OMPRT_NO_STACK (1u << 4)
/* Use the debug instantiation: assertions + call tracing compiled in, enabled at run time
 * by OMPRT_DEBUG (bit 0 assert, bit 1 trace) read at omprt_init. */
#define OMPRT_DEBUG_BUILD (1u << 5)
/* Generic mode: the region joins and the main thread runs a sequential postlogue. */
#define OMPRT_POSTLOGUE (1u << 6)
/* ICV probe: keep ICVs of nested data environments in thread ICV states. */
#define OMPRT_THREAD_STATES (1u << 7)
/* Fused variants: reduce the per-iteration verification inside the loop kernel instead of
 * storing it and summing with omprt_u64_sum (the paper moves the reduction out). */
#define OMPRT_FUSED_REDUCTION (1u << 8)
/* Testing only (omprt_spmd_axpy_sum): skip the host-side check of OMPRT_ASSUME_OVERSUB so
 * the debug build's device assertion ("asserting that the condition actually holds")
 * can be exercised.  In a release build a violated assumption then skips iterations. */
#define OMPRT_UNCHECKED (1u << 9)
/* omprt_xs_run_host: build and use the accelerated table layouts on the device (per call,
 * inside the end-to-end time). */
#define OMPRT_XS_ACCEL (1u << 10)
/* omprt_generic_team, NEXT f1 (P:174 SPMDization): the same target region in SPMD mode, the
 * sequential prologue guarded (thread 0) and broadcast by an aligned barrier; no state
 * machine.  inner_n <= 256. */
#define OMPRT_SPMDIZE (1u << 11)
/* omprt_generic_team, NEXT f2 (P:172 globalization elimination): generic mode with
 * the globalized arrays in static team-local shared memory -- no stack (0 B).  inner_n <= 256. */
#define OMPRT_DEGLOBALIZE (1u << 12)
/* (1u << 13) is unused: a per-thread bulk-copy SU(3) staging measured slower and removed. */
/* omprt_su3_mult / omprt_cuda_su3_mult: warp-cooperative staging -- a warp's 32 consecutive
 * site records (one contiguous 18 KiB range) are copied by coalesced 16 B cp.async into
 * padded shared-memory slots and written back by coalesced 16 B stores (one persistent team
 * of 192 per SM, per-warp double buffering); teams = 0: one per SM.  Not combined with
 * OMPRT_ASSUME_OVERSUB. */
#define OMPRT_WARP_STAGED (1u << 14)
/* omprt_xs_lookup / omprt_cuda_xs_lookup (B200 layouts required) and the e2e entry points:
 * flattened execution -- a persistent grid (teams = 0: the device's resident teams) whose
 * threads run their Fig. 5 iterations with the per-lookup nuclide loop fused into the
 * iteration loop (omprt::distribute_parallel_for_flat), so a SIMT lane that finishes its
 * lookup starts its next one instead of waiting for the warp's longest lookup.  Identical
 * results.  Not combined with OMPRT_ASSUME_OVERSUB or OMPRT_DEBUG_BUILD. */
#define OMPRT_XS_FLAT (1u << 15)
/* The same flag for omprt_rs_lookup / omprt_cuda_rs_lookup: persistent grid, one nuclide
 * of the material per flattened step (identical results to the nested form). */
#define OMPRT_FLAT OMPRT_XS_FLAT
/* With OMPRT_XS_FLAT: launch WITHOUT the L2 access-policy window that otherwise marks the
 * bracket records (t.brackets) persisting in the L2 set-aside granted by omprt_l2_set_aside
 * (cudaLimitPersistingL2CacheSize; without a set-aside there is no window either).
 * Persisting lines outlive the launch; omprt_l2_reset_persisting() returns them to
 * normal. */
#define OMPRT_XS_NO_L2_PERSIST (1u << 16)
/* schedule(dynamic, C) instead of Fig. 5's static assignment (reading R-D1): team t runs
 * the contiguous block [t*B, min(n, (t+1)*B)), B = ceil(n/teams), and its threads take
 * chunks of that block from a team-shared counter as they finish the previous one.  Same
 * per-iteration results; which thread runs an iteration is not deterministic.
 * omprt_spmd_axpy_sum_chunked (C = chunk) and, with OMPRT_FLAT, omprt_xs_lookup /
 * omprt_rs_lookup and their twins (C fixed per kernel). */
#define OMPRT_SCHED_DYNAMIC (1u << 17)
/* omprt_su3_mult / omprt_cuda_su3_mult: the site loop on a persistent grid with each warp's
 * 32 consecutive site records moved by ONE 2-D TMA tensor copy in (box [32][74] doubles:
 * the 2 columns past a 576 B record are zero-filled, giving padded 592 B shared-memory
 * slots) and one out (out-of-tensor columns are not written); double buffered per warp.
 * Not combined with OMPRT_ASSUME_OVERSUB or OMPRT_WARP_STAGED.  A and C
 * 16 B aligned. */
#define OMPRT_TMA_TILED (1u << 18)
/* omprt_spmd_axpy_sum / omprt_cuda_axpy_sum: the Fig. 5 loop with its operands moved by 2-D
 * TMA boxes -- b, c, a viewed as [n / (T*N)][T*N] matrices (row = trip, column = global
 * thread), each team streaming its N columns 16 trips per box, 4 boxes per array in
 * flight; the trailing partial trip from global memory.  Same iteration -> thread map and
 * per-thread order as Fig. 5 (a[] and the sum bit-identical).  threads <= 256 and a
 * multiple of 32; arrays 16 B aligned; no OMPRT_ASSUME_OVERSUB / OMPRT_DEBUG_BUILD. */
#define OMPRT_TMA_STREAM (1u << 19)
/* omprt_rs_lookup / omprt_cuda_rs_lookup with OMPRT_FLAT | OMPRT_SCHED_DYNAMIC: poles in the
 * Faddeeva function's Abrarov branch (|Z| < 6) are queued per warp in shared memory and
 * evaluated by all 32 lanes together (the runtime's lock-step warp-collective hook) instead
 * of by one divergent lane each; their contributions are added to the macroscopic cross
 * sections per pole (reading R-A8: a different summation order, within the RSBench
 * tolerance contract -- macro xs 1e-10 normwise, verification up to near-ties). */
#define OMPRT_RS_QUEUE (1u << 20)
/* (1u << 21) is unused: a warp-shared pole evaluation for RSBench measured slower. */

/* ---- runtime lifecycle ------------------------------------------------------------- */
typedef struct {
  uint64_t pool_bytes_per_team; /* global fallback slice per team (default 64 KiB) */
  uint64_t pool_teams;          /* teams covered by the pool (default 4096) */
  uint64_t max_teams;           /* capacity of the league-reduction partials (default 2^20) */
} omprt_options;

/* Create the per-device workspace; reads OMPRT_DEBUG.  opt may be NULL (defaults).
 * Idempotent per device.  Reserves NO L2 set-aside for persisting accesses (see
 * omprt_l2_set_aside: a reserved set-aside slows streaming kernels ~3x on B200). */
int omprt_init(int device, const omprt_options *opt);
int omprt_fini(int device);
/* Return every persisting L2 line of the current device's context to normal
 * (cudaCtxResetPersistingL2Cache; takes effect immediately, not stream-ordered: call it
 * with no launch in flight, e.g. before an L2 flush between timed steps). */
int omprt_l2_reset_persisting(void);
/* Resize the current device's L2 set-aside for persisting accesses to min(bytes, device
 * maximum) (synchronizes the device and resets persisting lines first); 0 removes it, and
 * the OMPRT_XS_FLAT launches then run without their access-policy window.  granted
 * (nullable) receives the size in effect. */
int omprt_l2_set_aside(uint64_t bytes, uint64_t *granted);
/* Device-side error recorded since init (0 = none); info (nullable) gets 4 ints
 * {team, thread, line, extra}. */
int omprt_device_status(int device, int *code, int *info);
/* Copies the calling thread's last error message (always NUL-terminated); returns its
 * length. */
int omprt_last_error(char *buf, size_t n);

/* Fig. 5 as a pure host function: the (team, thread) that runs iteration iv
 * of a combined distribute parallel for over n iterations.  OMPRT_E_INVAL if iv is not in
 * [0, n) or a size is not positive. */
int omprt_static_owner(int64_t iv, int64_t n, int32_t teams, int32_t threads, int32_t *team,
                       int32_t *thread);

/* ---- C1: SPMD axpy + fp64 sum (BASELINE configs[0]) -------------------------------- */
/* a[i] = fma(x, b[i], c[i]) for i in [0, n); *sum_inout += sum_i a[i] (team + league
 * reduction).  b, c, a: n doubles; sum_inout: 1 double; owner/count (nullable, test build
 * with OMPRT_RECORD_OWNER): n int32 each -- owner[i] = team*threads+thread, count[i] +=
 * 1.  flags: OMPRT_ASSUME_OVERSUB | OMPRT_RECORD_OWNER | OMPRT_DEBUG_BUILD. */
int omprt_spmd_axpy_sum(int64_t n, double x, const double *b, const double *c, double *a,
                        double *sum_inout, int32_t teams, int32_t threads, uint32_t flags,
                        int32_t *owner, int32_t *count, void *stream);
int omprt_cuda_axpy_sum(int64_t n, double x, const double *b, const double *c, double *a,
                        double *sum_inout, int32_t teams, int32_t threads, uint32_t flags,
                        int32_t *owner, int32_t *count, void *stream);

/* NEXT f3 -- C1 with a user chunk (Fig. 5 covers only "the absence of user-defined
 * chunks"): dist_schedule(static, chunk) + schedule(static, chunk) on the combined scheme,
 * chunk k = [k*chunk, min(n, (k+1)*chunk)) -> global thread k mod (teams*threads).  With
 * chunk = 4 and 32 B-aligned a, b, c each chunk moves with 256-bit accesses.
 * OMPRT_ASSUME_OVERSUB here means ceil(n/chunk) <= teams*threads.  Other arguments as
 * omprt_spmd_axpy_sum (owner[i] = owning global thread). */
int omprt_spmd_axpy_sum_chunked(int64_t n, int64_t chunk, double x, const double *b,
                                const double *c, double *a, double *sum_inout, int32_t teams,
                                int32_t threads, uint32_t flags, int32_t *owner, int32_t *count,
                                void *stream);
int omprt_cuda_axpy_sum_chunked(int64_t n, int64_t chunk, double x, const double *b,
                                const double *c, double *a, double *sum_inout, int32_t teams,
                                int32_t threads, uint32_t flags, int32_t *owner, int32_t *count,
                                void *stream);

/* ---- C2: generic-mode team kernel -------------------------------- */
/* Per team t: the main thread builds globalized w[inner_n], perm[inner_n] with
 * alloc_shared, then `parallel` + team `for` computes
 *   out[t*inner_n + j] = w[perm[j]] / s + w[j].
 * in/out: teams*inner_n doubles; owner (nullable): teams*inner_n int32 (OpenMP thread
 * number); postlogue (nullable, needs OMPRT_POSTLOGUE): teams doubles.  threads <= 1024,
 * inner_n <= 256 for the CUDA twin.  flags: OMPRT_GENERAL_SM | OMPRT_SMALL_STACK |
 * OMPRT_NO_STACK | OMPRT_POSTLOGUE | OMPRT_ASSUME_OVERSUB (inner_n <= threads) |
 * OMPRT_DEBUG_BUILD. */
int omprt_generic_team(int32_t teams, int32_t threads, int32_t inner_n, const double *in,
                       double *out, int32_t *owner, double *postlogue, uint32_t flags,
                       void *stream);
int omprt_cuda_generic_team(int32_t teams, int32_t threads, int32_t inner_n, const double *in,
                            double *out, int32_t *owner, double *postlogue, uint32_t flags,
                            void *stream);

/* ICV probe (Fig. 3/4): generic-mode kernel that records 7 int32 per query
 * point {thread_num, num_threads, level, active_level, in_parallel, team_num, num_teams}:
 * rec[t][0] prologue (main), rec[t][1+k] region thread k, rec[t][1+threads+k] inside a
 * nested parallel (num_threads(nested_request), serialized), rec[t][1+2*threads+k] after
 * it.  rec: teams*(1+3*threads)*7 int32.  flags: OMPRT_THREAD_STATES | OMPRT_DEBUG_BUILD |
 * OMPRT_GENERAL_SM. */
int omprt_icv_probe(int32_t teams, int32_t threads, int32_t nested_request, int32_t *rec,
                    uint32_t flags, void *stream);

/* Lock-step probe (tests): the lock-step flattened loop (Fig. 5 static, or dynamic with chunk
 * 3 when dynamic != 0) over n synthetic iterations, iteration i taking 1 + (7 i mod 13)
 * steps, with a body that uses the runtime's warp-collective hook.  steps[i] (n int32) gets
 * the steps iteration i ran, hooks[g] (teams*threads int32) how often the hook ran on
 * thread g; *errors (caller-zeroed int32) counts hook-contract violations (hook not on all
 * 32 lanes / not once per trip, done not reported exactly on an iteration's last step,
 * end() without it).  threads a multiple of 32. */
int omprt_lockstep_probe(int64_t n, int32_t teams, int32_t threads, int32_t dynamic,
                         int32_t *steps, int32_t *hooks, int32_t *errors, void *stream);

/* ---- C3: XSBench-shaped lookup (§V-A) ------------------------- */
typedef struct {
  const double *nuclide_grid; /* [n_isotopes*n_gridpoints][6] energy + 5 xs, per nuclide sorted */
  const double *unionized;    /* [n_union] sorted energies */
  const int32_t *index_grid;  /* [n_union][n_isotopes] lower bracket per nuclide */
  const int32_t *num_nucs;    /* [12] */
  const int32_t *mats;        /* [12][max_num_nucs] */
  const double *concs;        /* [12][max_num_nucs] */
  int32_t n_isotopes, n_gridpoints, max_num_nucs, pad;
  int64_t n_union;
  /* Optional B200 layouts of the same data, filled by omprt_xs_build_accel (all NULL: the
   * lookups read the tables above exactly as specified).  With them set the lookups read
   * the same values from: `bins` (search brackets of 2^log2_bins energy bins -- the same
   * unionized-grid index with ~4 instead of ~20 probes), `index_grid16` (the index grid as
   * uint16, n_gridpoints <= 65536: half the footprint, same values) and `brackets` (per
   * nuclide and bracket k the 12 doubles of gridpoints k and k+1, interleaved, 96 B per
   * bracket: 3 x 256-bit loads instead of 6 x 128-bit).  Results are identical. */
  const int32_t *bins;         /* [2^log2_bins + 1] */
  const uint16_t *index_grid16;/* [n_union][n_isotopes] */
  const double *brackets;      /* [n_isotopes][n_gridpoints-1][12], 32 B aligned */
  int32_t log2_bins, pad2;
} omprt_xs_tables;
/* Lookups first..first+count-1 (lookup i draws its energy and material from
 * fast_forward_LCG(seed, 2i), so results do not depend on sharding):
 * verification[i-first] = 1 + argmax of the 5 macroscopic cross sections (the first
 * maximum wins).  teams = 0: ceil(count/threads).  With OMPRT_FUSED_REDUCTION,
 * verification may be NULL and *checksum_inout += sum of the verification values instead
 * (checksum_inout device u64).  macro (nullable; test build, P:266 -- the values the
 * verification is the argmax of): [count][5] doubles, macro[(i-first)*5 + k] = macroscopic
 * xs k (total, elastic, absorption, fission, nu-fission), bit-identical to SURVEY App. A.1's
 * definition; written by a separate (unfused, release) instantiation of the same body, not
 * the timed one; OMPRT_E_INVAL with OMPRT_FUSED_REDUCTION or OMPRT_DEBUG_BUILD.
 * flags: OMPRT_ASSUME_OVERSUB | OMPRT_FUSED_REDUCTION | OMPRT_DEBUG_BUILD | OMPRT_XS_FLAT |
 * OMPRT_SCHED_DYNAMIC | OMPRT_XS_NO_L2_PERSIST. */
int omprt_xs_lookup(omprt_xs_tables t, uint64_t seed, int64_t first, int64_t count,
                    uint64_t *verification, uint64_t *checksum_inout, double *macro,
                    int32_t teams, int32_t threads, uint32_t flags, void *stream);
int omprt_cuda_xs_lookup(omprt_xs_tables t, uint64_t seed, int64_t first, int64_t count,
                         uint64_t *verification, uint64_t *checksum_inout, double *macro,
                         int32_t teams, int32_t threads, uint32_t flags, void *stream);
/* Byte sizes of the three accelerated-layout buffers for tables of this shape:
 * sizes[0] bins, sizes[1] index_grid16, sizes[2] brackets.  OMPRT_E_INVAL when
 * n_gridpoints > 65536 (the 16-bit index cannot hold it) or log2_bins not in [1, 28]. */
int omprt_xs_accel_sizes(int32_t n_isotopes, int32_t n_gridpoints, int64_t n_union,
                         int32_t log2_bins, uint64_t *sizes);
/* Build the accelerated layouts from t's device tables into caller-owned device buffers
 * (sizes from omprt_xs_accel_sizes; brackets 32 B aligned) on `stream`, and point t's
 * bins / index_grid16 / brackets / log2_bins at them.  A table-preparation step (like
 * XSBench's own index-grid construction), not part of a lookup. */
int omprt_xs_build_accel(omprt_xs_tables *t, int32_t *bins, uint16_t *index_grid16,
                         double *brackets, int32_t log2_bins, void *stream);
/* Derive XSBench's unionized energy grid and its index grid from the nuclide grids on the
 * device (XSBench builds them at initialization):
 *   unionized[e] = the e-th smallest of the n_isotopes*n_gridpoints energies
 *                  (nuclide_grid[i*6], i = nuclide*n_gridpoints + k; energies finite,
 *                  sorted within each nuclide, no -0.0),
 *   index_grid16[e*n_isotopes + q] = clip(#{k : E_q[k] <= unionized[e]} - 1, 0,
 *                  n_gridpoints - 2)   (ties handled exactly).
 * All pointers are device pointers (unionized: n_isotopes*n_gridpoints doubles,
 * index_grid16: that many rows of n_isotopes uint16); tmp: >= omprt_xs_derive_tmp_bytes
 * bytes of device scratch, 256 B aligned.  Asynchronous on `stream`.  OMPRT_E_INVAL
 * unless 0 < n_isotopes <= 4096 and 2 <= n_gridpoints <= 65536. */
int omprt_xs_derive_tmp_bytes(int32_t n_isotopes, int32_t n_gridpoints, uint64_t *bytes);
int omprt_xs_derive(const double *nuclide_grid, int32_t n_isotopes, int32_t n_gridpoints,
                    double *unionized, uint16_t *index_grid16, void *tmp, uint64_t tmp_bytes,
                    void *stream);
/* K11 ("we moved the reduction out of the timed kernel"): *out_inout += sum v[i]
 * (u64, wraps mod 2^64). */
int omprt_u64_sum(const uint64_t *v, int64_t n, uint64_t *out_inout, void *stream);
/* End-to-end offload with HOST tables (an OpenMP `target ... map(to: tables)
 * map(from: checksum)`): copies the tables host->device into library-owned buffers
 * (host pointers should be pinned), runs the lookups and the sum, and copies the u64
 * checksum back to *checksum_host.  Synchronous.  h2d_bytes/d2h_bytes (nullable) receive
 * the bytes moved. */
int omprt_xs_run_host(omprt_xs_tables host_tables, uint64_t seed, int64_t first, int64_t count,
                      int32_t threads, uint32_t flags, uint64_t *checksum_host,
                      uint64_t *h2d_bytes, uint64_t *d2h_bytes, void *stream);
/* The same offload repeated `steps` times (1..1024), each step with its own H2D of the
 * tables, lookups and D2H of its checksum (checksums_host[steps]); the H2D of step s+1 runs
 * on an internal copy stream while step s computes (two device table slots; OpenMP
 * `target nowait` + dependences).  host_tables may hold the B200 layouts on the host:
 * index_grid16 (then index_grid may be NULL and 2 B per entry cross PCIe) and/or brackets
 * (then nuclide_grid may be NULL); whatever is missing is built on the device (bins
 * always), which also enables the accelerated lookup (as OMPRT_XS_ACCEL does).  With
 * unionized, index_grid and index_grid16 all NULL only the raw problem data crosses PCIe
 * (nuclide_grid + materials) and the unionized grid and the 16-bit index grid are derived
 * on the device each step (omprt_xs_derive).  *h2d_bytes = bytes copied host->device per
 * step.  Synchronous. */
int omprt_xs_run_host_steps(omprt_xs_tables host_tables, uint64_t seed, int64_t first,
                            int64_t count, int32_t threads, uint32_t flags, int32_t steps,
                            uint64_t *checksums_host, uint64_t *h2d_bytes, uint64_t *d2h_bytes,
                            void *stream);

/* ---- C4: RSBench-shaped multipole lookup -------------------- */
typedef struct {
  /* [n_poles][8] EA RT RA RF (re, im), 32 B aligned -- in the lookups' PREPARED form (see
   * omprt_rs_prepare): EA.re / 2, (0 - EA.im) / 2, RT, RA, RF, sorted by l per window */
  const double *poles;
  const int32_t *pole_l;    /* [n_poles] l value in [0, numL); read by omprt_rs_prepare only */
  const double *windows;    /* [n_windows][4] T A F (prepared: l-run boundaries), 32 B aligned */
  const int32_t *win_range; /* [n_windows][2] absolute pole [start, end) */
  const int32_t *win_off;   /* [n_nuclides+1] window CSR offsets */
  const int32_t *n_windows; /* [n_nuclides] */
  const double *k0rs;       /* [n_nuclides][numL] */
  const int32_t *num_nucs;  /* [12] */
  const int32_t *mats;      /* [12][max_num_nucs] */
  const double *concs;      /* [12][max_num_nucs] */
  /* set by omprt_rs_prepare (NULL before): [n_mats][max_num_nucs][8] doubles per material
   * entry -- k0rs of its nuclide (4), conc, window offset | window count << 32 (bits), 2 pad */
  const double *matnuc;
  int32_t n_nuclides, numL, max_num_nucs;
  int32_t prepared; /* 1: poles, windows, matnuc hold the prepared form (omprt_rs_prepare) */
} omprt_rs_tables;
/* Table preparation (like omprt_xs_build_accel; not part of a lookup; App. A.2 defines the
 * lookup, this only lays its data out; n_mats = the number of materials of num_nucs / mats /
 * concs):
 * - prepared_poles (caller-owned device memory, n_poles * 8 doubles, 32 B aligned): the
 *   records of t->poles with EA replaced by (EA.re / 2, (0 - EA.im) / 2) -- exact in IEEE
 *   arithmetic; the lookup's Z = ((E - EA.re) / 2, (0 - EA.im) / 2) is then E/2 - EA.re/2
 *   and a load, the same bits, 3 fewer fp64 operations per pole (reading R-A9) -- and, within
 *   each window's range, stably sorted by the pole's l (reading R-A12: a window's poles are
 *   summed in l order, the same terms in another order);
 * - prepared_windows (caller-owned, n_windows * 4 doubles, 32 B aligned): T, A, F of each
 *   window and, as the 4th word, its l-run boundaries c1 | c2 << 21 | c3 << 42 (c_k = the
 *   number of the window's poles with l < k), so a lookup derives a pole's l from its index
 *   instead of loading pole_l;
 * - prepared_matnuc (caller-owned, n_mats * max_num_nucs * 8 doubles, 32 B aligned): one
 *   64 B record per material entry (m, j): k0rs of nuclide mats[m][j], concs[m][j], and
 *   win_off | n_windows << 32 of that nuclide (bit pattern), zeros past num_nucs[m]
 *   (reading R-A13: a nuclide step's 6-8 small loads become two).
 * Then points t->poles / t->windows / t->matnuc at them and sets t->prepared = 1.  Synchronizes
 * `stream` (the range checks come back to the host through a device workspace word: do not
 * run two omprt_rs_prepare calls on one device concurrently).  OMPRT_E_INVAL on null pointers, a
 * misaligned buffer, an already prepared table, numL != 4, a window range outside
 * [0, n_poles) or starting before the previous window's end (windows must not overlap), a
 * window of 2^21 poles or more, an l outside [0, 4), num_nucs outside [0, max_num_nucs],
 * a material entry outside [0, n_nuclides) or one whose nuclide's windows are not all among
 * the n_windows (a successful preparation makes every lookup's table access in-range); the
 * table is then unchanged. */
int omprt_rs_prepare(omprt_rs_tables *t, int64_t n_poles, int64_t n_windows, int32_t n_mats,
                     double *prepared_poles, double *prepared_windows,
                     double *prepared_matnuc, void *stream);
/* Same contract as omprt_xs_lookup (4 macroscopic cross sections; numL must be 4; the
 * tables prepared by omprt_rs_prepare, else OMPRT_E_INVAL).
 * macro (nullable): [count][4] doubles for parity tests. */
int omprt_rs_lookup(omprt_rs_tables t, uint64_t seed, int64_t first, int64_t count,
                    uint64_t *verification, double *macro, int32_t teams, int32_t threads,
                    uint32_t flags, void *stream);
int omprt_cuda_rs_lookup(omprt_rs_tables t, uint64_t seed, int64_t first, int64_t count,
                         uint64_t *verification, double *macro, int32_t teams, int32_t threads,
                         uint32_t flags, void *stream);

/* ---- C5: SU(3) link multiply -------------------------------------- */
/* C[s][l] = A[s][l] x B[l] (3x3 complex, fp64) for s in [0, n_sites); A, C: n_sites*72
 * doubles (site-major AoS), B: 72 doubles; *checksum_inout += sum of Re C (nullable).
 * teams = 0: ceil(n_sites/threads). */
int omprt_su3_mult(const double *A, const double *B, double *C, int64_t n_sites,
                   double *checksum_inout, int32_t teams, int32_t threads, uint32_t flags,
                   void *stream);
int omprt_cuda_su3_mult(const double *A, const double *B, double *C, int64_t n_sites,
                        double *checksum_inout, int32_t teams, int32_t threads, uint32_t flags,
                        void *stream);

/* ---- measurement probes (NOT the hot path): the roofs bench.py reports against ------- */
/* Read an L2-resident buffer (device, `bytes` >= 96, 32 B aligned; size it well below the
 * 126 MB L2) with 256-bit L1-non-allocating loads, the loads of the C3 bracket records:
 * mode 0 streams every 32 B sector `reps` times; mode 1 reads random 32 B sectors and mode 2
 * random 96 B records (3 adjacent sectors), `per_thread` (multiple of 8) per thread per
 * rep.  teams = 0: 2 per SM, 256 threads each.  The caller times the launch on `stream`.
 * sink: one device double (written only under a never-true condition). */
int omprt_probe_l2_read(const double *buf, uint64_t bytes, int32_t mode, int32_t reps,
                        int32_t per_thread, int32_t teams, double *sink, void *stream);
/* FP64 FMA throughput: `iters` steps of 8 independent fma chains per thread, 256 threads
 * per team, teams = 0: 8 per SM; flops = 16 * iters * teams * 256. */
int omprt_probe_fp64_fma(int64_t iters, int32_t teams, double *sink, void *stream);
/* HBM -> SM streaming bandwidth of `teams` SMs (1 <= teams <= the SM count): team b (32
 * threads, one per SM, 192 KB dynamic shared memory) reads its contiguous slice of `buf`
 * (device, 16 B aligned) by 16 KB bulk copies, 8 in flight; mode 1 also writes every second
 * chunk it read to `dst` (device, 16 B aligned, bytes / 2 writable), 2 bytes read per byte
 * written (C1's mix).  slice = floor(bytes / teams) rounded down to 32 KB (>= 32 KB, else
 * OMPRT_E_INVAL); bytes read = teams * slice, written = teams * slice / 2 in mode 1.  Size
 * `buf` above the 126 MB L2 so the reads come from HBM. */
int omprt_probe_hbm_stream(const void *buf, void *dst, uint64_t bytes, int32_t mode,
                           int32_t teams, double *sink, void *stream);

/* ---- introspection (resource report, "# Regs" and "SMem") ------------------ */
/* Number of kernels in the library and the name of kernel `id`. */
int omprt_kernel_count(void);
const char *omprt_kernel_name(int id);
/* cudaFuncGetAttributes of kernel `id`: registers per thread, static smem bytes, local
 * (spill/stack) bytes per thread, max threads per block. */
int omprt_kernel_attrs(int id, int *regs, int *static_smem, int *local_bytes,
                       int *max_threads);
/* Resident teams per SM of kernel `id` at `threads` per team and `dyn_smem` bytes of dynamic
 * shared memory (cudaOccupancyMaxActiveBlocksPerMultiprocessor): the theoretical occupancy
 * bench.py reports per config. */
int omprt_kernel_occupancy(int id, int threads, int dyn_smem, int *blocks_per_sm);

#ifdef __cplusplus
}
#endif
#endif /* OMPRT_H */
