/* include/cst.h — C ABI of libcst, the B200-native complex-stencil sweep + tuner.
 *
 * Paper: csTuner (Sun et al., IEEE CLUSTER 2021).  P:n = /root/reference/PAPER.md line n.
 * Problem statement followed by these calls (P:7): GIVEN a stencil
 * (pattern, order, coefficients, input grids), its grid and a parameterised combination of
 * optimisation techniques (Table I), RUN the stencil with a parameter setting
 * (cst_sweep) and DETERMINE the best-performing valid setting (cst_tune).
 *
 * Conventions (every function):
 *  - Returns cst_status; never throws, aborts or exits across the ABI.  On error the
 *    out-parameters are left untouched and cst_last_error() (thread-local) names the
 *    failing field or rule.
 *  - Device pointers are CUDA device addresses on the handle's device; host pointers are
 *    ordinary (preferably pinned) host memory.  The caller owns every buffer and stream;
 *    the library never frees caller memory.  Streams are passed as `void*` (a
 *    cudaStream_t / CUstream; NULL = legacy default stream) so C/ctypes callers need no
 *    CUDA headers.
 *  - A handle is not thread-safe; distinct handles are.
 *  - There is no CPU fallback: without a CUDA device every compute call returns
 *    CST_E_CUDA.
 */
#ifndef CST_H
#define CST_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  CST_OK = 0,
  CST_E_INVALID = 1,      /* malformed argument (null, overlap, bad layout, nsteps)       */
  CST_E_UNSUPPORTED = 2,  /* (kind, order) combination or feature not provided            */
  CST_E_CONSTRAINT = 3,   /* setting violates a rule R1..R13                */
  CST_E_CUDA = 4,         /* CUDA runtime/driver error (incl. no device)                   */
  CST_E_NVRTC = 5,        /* run-time compilation of a kernel variant failed               */
  CST_E_NCCL = 6,         /* NCCL error in the distributed sweep                           */
  CST_E_OOM = 7,          /* allocation failed                                             */
  CST_E_INTERNAL = 8
} cst_status;

const char* cst_status_str(cst_status s);
const char* cst_last_error(void);           /* thread-local detail of the last failure */
const char* cst_version(void);

/* ------------------------------------------------------------------ stencil + grid */
typedef enum { CST_STAR = 1, CST_BOX = 2, CST_HYPTERM = 3, CST_RHS4 = 4 } cst_kind;

/* Stencil spec "with order, coefficients and input grids" (north_star; P:13 order = the
 * neighbour extent along each dimension = radius r; Table III shapes).
 *   STAR    order 1..4, 1 in / 1 out, coeffs [c0, wx[-r..-1], wx[1..r], wy[..], wz[..]]
 *           (6r+1 values):  out = c0 u + sum_k wx[k] u(p+k ex) + (y) + (z)
 *   BOX     order 1, 1 in / 1 out, coeffs c[dz][dy][dx] z-major, (2r+1)^3 = 27 values
 *   HYPTERM order 4, 8 in (cons1..4, q1..4) / 5 out (flux0..4), coeffs
 *           [a1, a2, a3, a4, dxinv_x, dxinv_y, dxinv_z] (7 values); Table III "hypterm"
 *           (358 FLOPs, 13 I/O arrays) — definition in DESIGN.md §2.
 *   RHS4    order 2, 5 in (u1, u2, u3, mu, lambda) / 3 out (r1..r3), coeffs
 *           [s_x, s_y, s_z]: rhs4center-like variable-coefficient elastic operator
 *           (Table III "rhs4center", 666 FLOPs; SW4 [1]) — DESIGN.md §2 O7.
 * The coefficient array is copied at create time. */
typedef struct {
  int32_t kind;
  int32_t order;
  int32_t n_inputs;
  int32_t n_outputs;
  const double* coeffs;
  int32_t n_coeffs;
} cst_stencil_desc;

/* Padded, pitched FP64 grid; every array of one stencil shares it (element counts).
 * Element (x, y, z) with x, y, z in [-halo, n + halo) lives at
 *     base[((z + halo) * pitch_y + (y + halo)) * pitch_x + lead_x + x]
 * Requirements: halo >= order; lead_x >= halo; pitch_x >= lead_x + nx + halo and even;
 * pitch_y >= ny + 2*halo; base pointers 256-B aligned.  lead_x = 16 puts interior x = 0
 * on a 128-B boundary. */
typedef struct {
  int64_t nx, ny, nz;        /* updated interior points (nz = LOCAL planes for cst_dist) */
  int32_t halo;
  int32_t lead_x;
  int64_t pitch_x;
  int64_t pitch_y;
} cst_grid;

/* Parameter setting: Table I with the B200 extensions of DESIGN.md §3.
 * Encoding (Q14): bool/enum start at 1 with unit stride; numerics are powers of 2.
 * A zero-initialised struct is NOT valid: start from cst_setting_default or cst_space_at. */
typedef struct {
  int32_t tb[3];          /* TB_x, TB_y, TB_z: CTA shape */
  int32_t staging;        /* 1 none (L1/L2), 2 smem ld/st, 3 smem via TMA */
  int32_t use_constant;   /* 1 coefficients as kernel params, 2 __constant__ */
  int32_t use_streaming;  /* 1 off (3-D tiles), 2 2.5-D streaming */
  int32_t sd;             /* streaming dim 1 x, 2 y, 3 z; 1 when streaming off */
  int32_t sb;             /* concurrent-streaming chunk (planes); 1 when off */
  int32_t uf[3];          /* loop unrolling factors */
  int32_t cm[3];          /* cyclic merging (points at stride TB_d*BM_d) */
  int32_t bm[3];          /* block merging (adjacent points) */
  int32_t use_retiming;   /* 1 gather form, 2 retimed scatter accumulation
                           * Rule R16 (rhs4): 2 selects the retimed column walk (outer-s
                           * products scattered to pending outputs, inner-s product planes;
                           * DESIGN.md §4.5) and needs streaming with T_SD = 1, TMA staging,
                           * bt = 1, CM = 1, BM_b = 1, BM_x <= 2. */
  int32_t prefetch;       /* 1 off, 2..4 pipeline stages in flight */
  int32_t bt;             /* temporal blocking degree {1,2,4}: sweeps fused per kernel
                           * pass (B200 extension, "more
                           * optimization parameters").  Rule R14: bt > 1 needs star/box,
                           * z streaming with T_z = 1, TMA staging, retiming, CM = UF = 1,
                           * BM_x, BM_y <= 2.  Only matters for nsteps > 1 (cst_sweep). */
  int32_t qstore;         /* where the streamed-direction state lives {1 registers, 2 tensor
                           * memory (TMEM)}: B200 extension of retiming — a ring of R
                           * (value, partial output) pairs per point in TMEM frees the
                           * registers for larger register blocks.  Rule
                           * R15: qstore = 2 needs the star or hypterm (hypterm: one point
                           * along x, BM_b <= 2, CM = 1), streaming with T_SD = 1, TMA
                           * staging, retiming, bt = 1, and ceil(threads/128) * points per
                           * thread * (4r star, 20r hypterm) <= 512 TMEM columns; or rhs4's
                           * retimed walk (R16), whose s-window queue then takes 10 (2r + 1)
                           * columns per point. */
} cst_setting;

typedef struct cst_stencil cst_stencil;     /* opaque: JIT modules, TMA descriptors, space */

/* Create a handle for (stencil, grid) on CUDA device `device`.  Validates the desc and
 * grid (CST_E_INVALID / CST_E_UNSUPPORTED); does not need a GPU until the first sweep. */
cst_status cst_stencil_create(const cst_stencil_desc* desc, const cst_grid* grid, int device,
                              cst_stencil** out);
void cst_stencil_destroy(cst_stencil* h);

/* Rules R1-R12, R14-R16 (explicit, implicit analytic resource rules, P:149-151,
 * and the structural rules of the B200 extensions).
 * CST_OK if valid, else CST_E_CONSTRAINT with the rule in cst_last_error(). */
cst_status cst_setting_check(const cst_stencil* h, const cst_setting* s);
/* A good default setting for the handle's stencil (valid by construction). */
cst_status cst_setting_default(const cst_stencil* h, cst_setting* s);

/* Canonical valid space: lexicographic order of the 21 fields (Table I row order, bt, qstore;
 * values ascending) restricted to valid tuples; rank = position (bit-exact with
 * oracle/space.py). */
cst_status cst_space_count(cst_stencil* h, uint64_t* n);
cst_status cst_space_at(cst_stencil* h, uint64_t rank, cst_setting* s);
cst_status cst_space_rank(cst_stencil* h, const cst_setting* s, uint64_t* rank);

/* Compiled-variant facts (compiles on first use).  Used by the tuner's static features. */
typedef struct {
  int32_t registers;       /* per thread                         */
  int32_t local_bytes;     /* stack frame + spill (0 required)   */
  int32_t smem_bytes;      /* dynamic shared memory per CTA      */
  int32_t threads;         /* per CTA                            */
  int32_t ctas_per_sm;     /* occupancy (cudaOccupancy...)       */
  int64_t grid_ctas;       /* CTAs launched per sweep            */
  double compile_s;        /* NVRTC time of this variant (0 on a cache hit) */
} cst_kernel_info;
cst_status cst_kernel_info_get(cst_stencil* h, const cst_setting* s, cst_kernel_info* info);
/* Code generation only: generate and NVRTC-compile the sm_100a variant of a valid
 * setting into the cubin cache; needs no GPU.  *compile_s = seconds (0 on a cache hit). */
cst_status cst_variant_compile(const cst_stencil* h, const cst_setting* s, double* compile_s);
/* The generated code itself: copy the sm_100a cubin of a valid setting's variant
 * (compiled if needed; no GPU) into buf[cap].  *size = cubin bytes, always set; if cap is
 * smaller than that nothing is copied and CST_E_INVALID is returned (call with cap = 0 to
 * size the buffer).  remote = 1 selects the fused-halo twin (CST_REMOTE).  Used to audit
 * that distinct settings generate distinct code (tests/test_codegen_distinct.py). */
cst_status cst_variant_cubin(const cst_stencil* h, const cst_setting* s, int32_t remote,
                             void* buf, int64_t cap, int64_t* size);

/* One sweep (nsteps = 1) or nsteps ping-pong sweeps over DEVICE buffers, asynchronous on
 * `stream`.  in[n_inputs], out[n_outputs].  nsteps = 1: only interior points of out[] are
 * written, output halos are never touched.  nsteps > 1 requires n_inputs == n_outputs
 * (ping-pong: the interior of in[] is overwritten; result in out if nsteps is odd, else in
 * in); in[]'s halo is the boundary condition of every step and is first copied into
 * out[]'s halo (reading Q23).  With s->bt > 1 the steps run as kernel passes of
 * up to bt fused sweeps (temporal blocking); the pass count keeps nsteps' parity, so the
 * result placement is the same for every bt.  Inputs must not overlap outputs
 * (CST_E_INVALID).  Allocates nothing after first use. */
cst_status cst_sweep(cst_stencil* h, const cst_setting* s, const double* const* in,
                     double* const* out, int32_t nsteps, void* stream);
/* Same computation over HOST buffers (end-to-end path): copies the inputs host->device,
 * sweeps, copies the outputs device->host, synchronises.  Device staging buffers are
 * owned by the handle (allocated on first use, reused). */
cst_status cst_sweep_host(cst_stencil* h, const cst_setting* s, const double* const* in,
                          double* const* out, int32_t nsteps);
/* Wait for the handle's work and surface asynchronous kernel errors. */
cst_status cst_sync(cst_stencil* h);

/* Number of kernel launches the last cst_sweep/cst_sweep_host issued. */
int64_t cst_last_launch_count(const cst_stencil* h);

/* Fill the logical region [-halo, n+halo)^3 of a device grid with the cstgen generator
 * (cstgen/cst_gen.h): value(seed, array_id, global padded index over an
 * (nx_global, ny_global) x-y extent), local plane z maps to global z + z0.  Pad columns
 * get `pad_value`.  Asynchronous on `stream`. */
cst_status cst_fill_uniform(const cst_grid* g, double* dev, uint64_t seed, uint64_t array_id,
                            int64_t nx_global, int64_t ny_global, int64_t z0,
                            double pad_value, void* stream);

/* Time a setting: `warmup` untimed cst_sweep calls of `nsteps` steps, then the median of
 * `reps` CUDA-event timed calls on `stream` (fitness of P:351 / Q20).  *ms = median
 * milliseconds PER STEP (call time / nsteps).  nsteps > 1 overwrites in[] (ping-pong). */
cst_status cst_time_setting(cst_stencil* h, const cst_setting* s, const double* const* in,
                            double* const* out, int32_t nsteps, int32_t warmup, int32_t reps,
                            void* stream, double* ms);

/* Hardware counters of one sweep (CUPTI range profiler, user range + user replay: the
 * sweep is re-run once per counter pass).  names: metric names as ncu / CUPTI spell them
 * (e.g. "dram__bytes_read.sum"); values[n] receives their GPU values.  CST_E_UNSUPPORTED
 * when libcupti is missing or counters are not permitted.  (the paper
 * collects its dataset's GPU metrics with Nsight.) */
cst_status cst_collect_metrics(cst_stencil* h, const cst_setting* s, const double* const* in,
                               double* const* out, const char* const* names, int32_t n,
                               double* values);

/* FP64 FMA throughput of the device (TFLOP/s, 2 FLOPs per DFMA), measured by a DFMA-chain
 * microbenchmark: the FP64 roofline denominator.  *sm_clock_ghz = the device's max clock. */
cst_status cst_fp64_peak(int device, double* tflops, double* sm_clock_ghz);

/* ------------------------------------------------------------------------ tuner */
/* csTuner method: dataset, CV + Algorithm 1 grouping
 * (P:155-230), PCC + Algorithm 2 metric combination, PMNF surrogate + RSE
 * (Eq. 3), threshold sampling, re-indexing, grouped
 * multi-population GA with CV_top-n approximation stop.  Defaults = paper
 * values where the paper gives one. */
typedef struct {
  uint64_t seed;
  int32_t dataset_size;      /* 128 */
  double sampling_ratio;     /* 0.10 */
  int32_t n_subpops;         /* 2 */
  int32_t subpop_size;       /* 16 */
  double crossover;          /* 0.8 */
  double mutation;           /* 0.005 */
  int32_t top_n;             /* 10 (Fig. 4)                              */
  double cv_threshold;       /* 0.02                                            */
  int32_t max_generations;   /* 50 per group                                    */
  int32_t num_collections;   /* 3                                               */
  double time_budget_s;      /* 100: search time after the dataset (its
                                metric collection is offline); <= 0 = none    */
  int32_t reps;              /* timed reps per evaluation (median)              */
  int32_t warmup;            /* untimed sweeps per evaluation                   */
  const char* log_path;      /* JSON report of every stage, or NULL              */
  int32_t n_user_metrics;    /* metrics supplied by the eval callback (0 = model) */
  int32_t quantile_sample;   /* settings sampled to set thresholds / gene tables  */
  int32_t warm_start;        /* 1: add cst_setting_default() to the dataset (ours) */
  int32_t metrics_mode;      /* 0: CUPTI counters for the dataset if available, else
                                modelled features; 1: modelled features only        */
  int32_t nsteps;            /* steps per cst_sweep call of the tuned workload (1); the
                                fitness is ms per step.  With nsteps = 1 a setting is
                                timed as its bt = 1 twin; with nsteps > 1 the built-in
                                evaluator times ping-pong on its own device copies   */
  int32_t noise_reps;        /* 8: re-evaluate the dataset's best setting this many
                                times; the CV of those fitness values (timing noise)
                                sets the approximation threshold to
                                max(cv_threshold, 2 * noise CV) (Q18); 0 =
                                cv_threshold as given                                */
  int32_t filter_threads;    /* host threads streaming the whole valid space through
                                the PMNF threshold filter (0 = all cores)             */
  int32_t cool_ms;           /* 30: idle ms before each built-in timing, so every
                                candidate is timed in the same (boost-clock) power
                                state instead of later ones under the board's power
                                cap                                   */
} cst_tune_opts;

typedef struct {
  double best_ms;            /* median ms of the best setting                   */
  double best_gstencils;     /* interior points / best time                     */
  uint64_t space_count;      /* valid settings                                   */
  uint64_t sampled_count;    /* settings of the whole valid space kept by the PMNF
                                threshold filter (counted exactly)        */
  uint64_t evaluations;      /* distinct settings timed (incl. dataset)          */
  uint64_t jit_compiles;
  double wall_s, eval_s, jit_s, preproc_s;
  int32_t n_groups;
  int32_t generations;
  int32_t phases_cv_stop;    /* GA phases ended by the CV_top-n approximation */
  double noise_cv;           /* CV of the noise_reps re-evaluations (0 if none)      */
  double cv_threshold_used;  /* the approximation threshold applied               */
} cst_tune_report;

void cst_tune_opts_default(cst_tune_opts* o);

/* Evaluation callback: fitness of `n` candidate settings (e.g. spread over GPUs by the
 * caller — population-parallel evaluation).  Must write ms[i] (> 0, or
 * <= 0 / inf for an invalid or failed candidate).  If opts->n_user_metrics > 0 it must
 * also write metrics[i * n_user_metrics + k] (the dataset's "GPU metrics");
 * otherwise metrics is NULL and the tuner uses its modelled features.
 * Returns 0 on success. */
typedef int (*cst_eval_fn)(void* user, const cst_setting* settings, int32_t n, double* ms,
                           double* metrics);

cst_status cst_tune(cst_stencil* h, const cst_tune_opts* o, const double* const* in,
                    double* const* scratch_out, cst_eval_fn eval, void* eval_user,
                    cst_setting* best, cst_tune_report* rep);

/* ------------------------------------------------------------------ distributed */
/* z-slab domain decomposition: rank k owns global interior planes
 * [k*nz, (k+1)*nz) of a grid of nranks*nz planes, nz = the handle's grid.nz.  Each step:
 * boundary planes first, then the halo exchange (r planes to/from rank +-1) on a
 * communication stream concurrently with the interior planes.  Physical z-end halos are
 * caller data.  Transport: NCCL (nccl_unique_id = 128-byte ncclUniqueId broadcast by the
 * caller, e.g. through torch.distributed), or, with nccl_unique_id == NULL, the fused
 * peer-memory transport below (one process per GPU); cst_dist_sweep_loopback drives all
 * slabs from one process on one device (cudaMemcpyAsync) to test the decomposition. */
typedef struct cst_dist cst_dist;

/* Halo-exchange plan of rank `rank` in a z-slab decomposition over `nranks` ranks, each
 * owning `nz` local planes, stencil radius `r`: up to 4 transfers of r contiguous planes
 * (send local planes [0, r) to rank-1 / [nz-r, nz) to rank+1; receive into halo planes
 * [-r, 0) from rank-1 / [nz, nz+r) from rank+1).  plane_begin is a LOCAL interior z
 * (negative = halo).  Used by cst_dist_sweep, the loopback transport and the CPU tests. */
typedef struct {
  int32_t peer;          /* rank on the other side                         */
  int32_t is_send;       /* 1 send, 0 receive                               */
  int64_t plane_begin;   /* first local plane (interior z coordinate)       */
  int64_t nplanes;       /* = r                                              */
} cst_halo_xfer;
cst_status cst_dist_halo_plan(int32_t nranks, int32_t rank, int64_t nz, int32_t r,
                              cst_halo_xfer* xfers /* [4] */, int32_t* n_xfers);
cst_status cst_dist_create(cst_stencil* h, int32_t nranks, int32_t rank,
                           const void* nccl_unique_id, cst_dist** out);
cst_status cst_dist_nccl_unique_id(void* id128);        /* ncclGetUniqueId */
cst_status cst_dist_sweep(cst_dist* d, const cst_setting* s, const double* const* in,
                          double* const* out, int32_t nsteps, void* stream);
/* Loopback: one process drives all slabs; in_slabs[k*n_inputs + a], out likewise. */
cst_status cst_dist_sweep_loopback(cst_stencil* h, int32_t nslabs, const cst_setting* s,
                                   double* const* in_slabs, double* const* out_slabs,
                                   int32_t nsteps, void* stream);
void cst_dist_destroy(cst_dist* d);

/* ---------------------------------------------------- population-parallel tuning */
/* cst_tune with each GA population (and the dataset) evaluated across the ranks of a
 * cst_dist (the paper's multi-process GA): rank 0 runs the tuner
 * (every stage of cst_tune, same options, same result for the same fitness values); every
 * batch of candidates it asks for is broadcast, rank k evaluates candidates i with
 * i % nranks == k on its own GPU, and the fitness (and metric) vectors are all-gathered.
 * The GA's trajectory therefore does not depend on nranks.  COLLECTIVE: every rank of `d`
 * calls it with the same opts.
 *   in / scratch_out: this rank's replica of the evaluation grid (device buffers of the
 *     handle's grid), used by the built-in evaluator (NVRTC code generation of the share
 *     on host threads, then CUDA-event timing, Q20) when local_eval == NULL;
 *   local_eval: optional caller evaluation of this rank's share (same contract as
 *     cst_tune's eval callback; synthetic objectives in the tests);
 *   best / rep: written on every rank (rank 0's result is broadcast); rep->evaluations
 *     etc. are rank 0's.
 * Transport: the handle's NCCL communicator (small device staging buffers on its
 * communication stream), or the host collectives given to cst_dist_create_host.  Errors:
 * if rank 0's tuner fails, every rank returns that status (the result message is always
 * broadcast, so no rank blocks); a rank whose evaluation fails reports its candidates as
 * invalid (fitness 0) and keeps serving. */
typedef struct {
  void* user;
  /* broadcast `bytes` of host memory at buf from rank `root` (in place); 0 = success */
  int (*bcast)(void* user, void* buf, int64_t bytes, int32_t root);
  /* all-gather `bytes` from every rank: recv[k * bytes ...] = rank k's send; 0 = success */
  int (*allgather)(void* user, const void* send, void* recv, int64_t bytes);
} cst_collectives;
/* A tuning-only handle (no device resources; cst_dist_sweep on it is CST_E_INVALID) whose
 * collectives are the caller's (e.g. torch.distributed over gloo or NCCL).  `coll` is
 * copied; its user pointer must stay valid for the handle's lifetime. */
cst_status cst_dist_create_host(cst_stencil* h, int32_t nranks, int32_t rank,
                                const cst_collectives* coll, cst_dist** out);
cst_status cst_dist_tune(cst_dist* d, const cst_tune_opts* o, const double* const* in,
                         double* const* scratch_out, cst_eval_fn local_eval, void* local_user,
                         cst_setting* best, cst_tune_report* rep);

/* Fused halo exchange over peer memory (no NCCL).  A handle created
 * with nccl_unique_id == NULL and nranks > 1 uses it: the boundary kernels of
 * cst_dist_sweep store every edge-plane value both locally and, through a CUDA IPC
 * mapping, straight into the neighbour's halo (NVLink / NVSwitch peer stores), and the
 * ranks order their steps with flag words written over the same mappings (release /
 * acquire, system scope; a wait gives up after 30 s with a device trap instead of hanging).
 * Setup, once per pair of ping-pong buffer sets (a = in[] of the first call, b = out[]):
 *   cst_dist_p2p_export(d, a, b, blob)   writes CST_P2P_BLOB_BYTES describing my buffers
 *                                         and flag words (IPC handles + offsets)
 *   the caller exchanges blobs (e.g. torch.distributed.all_gather_object)
 *   cst_dist_p2p_import(d, peer, blob)   for peer = rank - 1 and rank + 1 (if they exist)
 * cst_dist_sweep then requires {in, out} to be {a, b} in either order (CST_E_INVALID
 * otherwise).  Buffers must come from cudaMalloc (any caching allocator built on it). */
#define CST_P2P_BLOB_BYTES 2048
cst_status cst_dist_p2p_export(cst_dist* d, double* const* buf_a, double* const* buf_b,
                               void* blob);
cst_status cst_dist_p2p_import(cst_dist* d, int32_t peer, const void* blob);

#ifdef __cplusplus
}
#endif
#endif /* CST_H */
