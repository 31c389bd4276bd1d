/*
 * stencilfuse.h — C ABI of the B200-native stencil-DAG executor.
 *
 * The hot path of Wahib & Maruyama, "Automated GPU Kernel Transformations in
 * Large-Scale Production Stencil Applications" (HPDC'15; /root/reference/PAPER.md,
 * cited P:L<line> §<section>): a stencil application is a sequence of
 * memory-bound kernels over shared 3-D arrays (§1, §2); the method
 * replaces them by fused kernels that keep intermediates on chip with halo
 * recompute (complex fusion, §5.5.3), input sharing (simple fusion,
 * P:L288 §5.5.2), after optional fission of kernels into independent pieces
 * (§4.1, Algorithm 2).  This library executes a program either as
 * written (run_unfused, "no fusion" P:L284 §5.5.1) or under a fission/fusion
 * plan (run_fused, host invocation order P:L296 §5.5.4), on one GPU or on a
 * z-slab decomposition over several GPUs (exchange_halos).
 *
 * Conventions
 *  - Every function returns sp_status; SP_OK == 0.  On error a message is
 *    available from sp_last_error() (thread-local, valid until the next call
 *    on the same thread).  No C++ exception crosses this boundary.
 *  - Host pointers are read during the call only; the library deep-copies
 *    every description it is given.
 *  - Device pointers are borrowed (stencil_program_bind): the caller owns the
 *    memory and keeps it alive while the program may use it.
 *  - cudaStream_t arguments are borrowed; run_* and exchange_halos are
 *    asynchronous and stream-ordered.  Launch errors are reported
 *    synchronously; asynchronous faults surface at the caller's next sync.
 *  - A handle is not thread-safe; distinct handles are independent.
 *  - Nothing here falls back to the CPU: without a usable CUDA device the
 *    device entry points return SP_E_CUDA.
 */
#ifndef STENCILFUSE_H
#define STENCILFUSE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *sp_stream; /* == cudaStream_t */

typedef enum {
    SP_OK = 0,
    SP_E_ARG = 1,            /* bad argument, size or index                          */
    SP_E_PROGRAM = 2,        /* program violates the model (R3 race, tap > ghost ...) */
    SP_E_PLAN_PARTITION = 3, /* a statement missing or listed twice                  */
    SP_E_PLAN_ORDER = 4,     /* a dependency edge points backwards in the plan       */
    SP_E_PLAN_HAZARD = 5,    /* a group reads from HBM an array it also stores (R11) */
    SP_E_RESOURCES = 6,      /* no tile fits shared memory / halo deeper than alloc  */
    SP_E_JIT = 7,            /* NVRTC compilation or module load failed              */
    SP_E_CUDA = 8,           /* CUDA runtime/driver error (or no device)             */
    SP_E_NCCL = 9,           /* NCCL error                                           */
    SP_E_STATE = 10          /* call not valid in the current state                  */
} sp_status;

typedef enum { SP_F32 = 4, SP_F64 = 8 } sp_dtype; /* value = element size in bytes */

/* Array roles.  IN: read only.  OUT/INOUT: results compared after a run
 * (INOUT may also be read first).  TEMP: inter-kernel intermediate whose HBM
 * content after run_fused is unspecified (reading R6 in DESIGN.md). */
typedef enum { SP_IN = 1, SP_OUT = 2, SP_INOUT = 3, SP_TEMP = 4 } sp_role;

/* One access a[p + (dx,dy,dz)]; |d| must not exceed the ghost width. */
typedef struct { int32_t array, dx, dy, dz; } sp_tap;

/* term = coef * a[p+da]            (has_b == 0)
 *      = (coef * a[p+da]) * b[p+db] (has_b != 0)                       (R4) */
typedef struct { double coef; sp_tap a; int32_t has_b; sp_tap b; } sp_term;

/* out[p] = term0 + term1 + ... accumulated left to right, for every interior p
 * (the stencil operations of the paper's "operations metadata", §3.2.1). */
typedef struct { int32_t out; int32_t n_terms; const sp_term *terms; } sp_stmt;

/* A kernel: ordered statements executed per point (reading R3:
 * an array written by the kernel may be read by it only at offset 0).
 * box: the kernel's loop bounds (§5.5.2, kernels with "shorter loops",
 * e.g. boundary kernels on one plane): NULL = the whole interior,
 * else 6 values {x0, x1, y0, y1, z0, z1}, half-open, in GLOBAL interior
 * coordinates, 0 <= x0 <= x1 <= nx, 0 <= y0 <= y1 <= ny, 0 <= z0 <= z1 <=
 * nz_global (copied at create time).  The kernel's statements write exactly
 * the interior points inside the box; every other point of their output
 * arrays keeps its stored value (reading R2').  SP_E_PROGRAM if out of range. */
typedef struct {
    const char *name;
    int32_t n_stmts;
    const sp_stmt *stmts;
    const int64_t *box;
} sp_kernel;

typedef struct { const char *name; sp_role role; } sp_array_desc;

/* Grid of THIS process.  z is the marched and the decomposed axis.
 *   nx, ny      interior size in x (contiguous) and y
 *   nz_local    interior planes owned by this rank
 *   nz_global   interior planes of the whole grid (== nz_local on one rank)
 *   z_offset    global z of local plane 0
 *   ghost[3]    ghost width per axis (>= max |offset| of any tap)
 *   zhalo       ghost planes allocated below/above in z (>= ghost[2]); the
 *               deep halo that fused groups with accumulated z-reach need on
 *               several ranks.  0 means ghost[2]. */
typedef struct {
    int64_t nx, ny, nz_local, nz_global, z_offset;
    int32_t ghost[3];
    int32_t zhalo;
    sp_dtype dtype;
} sp_grid;

typedef struct { int32_t kernel, stmt; } sp_stmt_ref;

/* Storage of every array (identical for all arrays of a program):
 * dense [z_alloc][y_alloc][x_pitch] elements, x fastest; interior point
 * (i,j,k) at ((k+origin_z)*y_alloc + j+origin_y)*x_pitch + i+origin_x.
 * x_pitch*elem is a multiple of 128 B; base pointers must be 256-B aligned. */
typedef struct {
    int64_t x_pitch, y_alloc, z_alloc, origin_x, origin_y, origin_z, bytes;
} sp_layout;

/* DDG/OEG edge between statements (global statement ids in program order,
 * P:L104-136 §3.2.3; reading R9/R10).  kind: bit0 RAW, bit1 WAR, bit2 WAW. */
typedef struct { int32_t from, to, kind, array; } sp_edge;

/* Per-launch report of a group (fused) or kernel (unfused).  Byte/flop figures
 * are per interior grid point of one launch.                              */
typedef struct {
    int32_t n_stmts;          /* statements computed (dead ones excluded)        */
    int32_t n_inputs;         /* arrays read from HBM (ExtIn)                    */
    int32_t n_stores;         /* arrays written to HBM (LiveOut, reading R6)      */
    int32_t n_smem_stages;    /* on-chip stages kept in shared-memory planes      */
    int32_t n_reg_stages;     /* on-chip stages kept in registers / queues        */
    int32_t ext[4];           /* max halo extension of any stage: x-, x+, y-, y+  */
    int32_t z_below, z_above; /* planes read below/above the output plane (reach) */
    int32_t tile_x, tile_y, zchunk, threads;
    int32_t grid_ctas;        /* CTAs per launch                                 */
    int32_t regs_per_thread;  /* after JIT (-1 before)                           */
    int64_t smem_bytes;       /* dynamic shared memory per CTA                   */
    double bytes_alg;         /* elem * (|ExtIn| + |LiveOut|)                    */
    double flops_alg;         /* sum over stmts of 2*terms - 1 + products         */
    double bytes_exec;        /* incl. halo re-reads and z warm-up planes         */
    double flops_exec;        /* incl. halo recompute and warm-up                 */
    double smem_bytes_pt;     /* shared-memory traffic per point (model)          */
    int32_t block_x, block_y, block_cby; /* per-thread register block of the core  */
    double t_model_us;        /* modelled launch time (tile chooser objective)    */
    int32_t zqueue;           /* z-reuse policy in effect (the option's values)  */
    int32_t est_regs;         /* registers per thread the chooser assumed        */
    int32_t warmup_steps;     /* z steps a chunk runs before its first plane      */
    int32_t prefetch;         /* TMA batches in flight ahead of the compute warps */
    double instr_pt;          /* modelled issued instructions per point (thread)  */
} sp_group_report;

typedef struct sp_comm_s sp_comm;
typedef struct stencil_program_s stencil_program;

/* ---- communicator (z-slab decomposition) -------------- */
/* nccl_unique_id: the 128-byte ncclUniqueId produced by rank 0 (sp_comm_unique_id)
 * and broadcast by the caller (e.g. torch.distributed).  The current CUDA
 * device of the calling thread is used.  Collective over nranks. */
sp_status sp_comm_unique_id(void *out128);
sp_status sp_comm_create(const void *nccl_unique_id, int32_t nranks, int32_t rank, sp_comm **out);
/* Test transport: nranks communicators (out[0..nranks-1]) of in-process virtual
 * ranks on the current device.  Each virtual rank's program must be driven from
 * its own host thread (the exchanges meet at host barriers, 120 s timeout ->
 * SP_E_STATE); ghost planes are pulled from the neighbours' bound slabs with
 * device-to-device copies on the comm stream, ordered by events, in place of
 * ncclSend/ncclRecv.  Every other step of the multi-rank schedule (exchange set,
 * interior/boundary planes, events) is the NCCL path's.  Destroy each with
 * sp_comm_destroy. */
sp_status sp_comm_create_loopback(int32_t nranks, sp_comm **out);

/* ---- peer-push halo exchange (option "xpush" = 1, several ranks) ----------
 * SURVEY.md §8(e) "B200-native step beyond send/recv" / §8(f) NEXT #2.  With
 * the option set, an epoch of a TEMP array that begins at a store (see
 * sp_plan_exchange) is not exchanged by the communicator: the storing kernel
 * writes the bottom/top planes the neighbours' readers need straight into the
 * neighbours' ghost planes (st.global to peer memory over NVLink/NVSwitch), and
 * every kernel of the rank runs a progress protocol with its neighbours: chunks
 * within reach of a slab end wait (in the kernel) until both neighbours have
 * completed the previous launch, and the last CTA of each kernel publishes its
 * completion to both neighbours (fence.sc.sys + st.release.sys).  Step-start
 * epochs (IN arrays, previous-step state) still travel through the communicator.
 * Every rank must bind, before its first run:
 *   - sp_bind_peer(array, side, ptr) for each TEMP array: the neighbour's buffer
 *     of that array (side 0 = rank-1, 1 = rank+1) mapped in this process;
 *   - sp_bind_peer_signal(side, ptr): the neighbour's signal block
 *     (sp_signal_buffer on that rank, 64 B of device memory it owns).
 * Unbound neighbours of an existing side give SP_E_STATE at the run.  A rank
 * that stops running makes its neighbours' waiting kernels trap after 20 s
 * (no hang).  Layouts must be identical on all ranks (same grid and zhalo). */
sp_status sp_signal_buffer(stencil_program *prog, void **out);
sp_status sp_bind_peer(stencil_program *prog, int32_t array, int32_t side, void *peer_ptr);
sp_status sp_bind_peer_signal(stencil_program *prog, int32_t side, void *peer_signal);
/* CUDA IPC of a device pointer (any pointer inside a cudaMalloc allocation, e.g.
 * a torch tensor): 64-byte handle of the allocation + the pointer's offset in it.
 * sp_ipc_open maps it in another process (once per allocation; mappings live
 * until the process exits).  SP_E_CUDA on failure. */
sp_status sp_ipc_export(const void *dev_ptr, void *handle64, int64_t *offset);
sp_status sp_ipc_open(const void *handle64, int64_t offset, void **dev_ptr);
void sp_comm_destroy(sp_comm *comm);

/* ---- program ------------------------------------------------------------ */
/* Validates and deep-copies the program (kernels in host invocation order,
 * P:L136).  comm may be NULL (single rank).  Errors: SP_E_ARG (sizes),
 * SP_E_PROGRAM (tap beyond ghost, unknown array, R3 in-kernel race,
 * statement without terms). */
sp_status stencil_program_create(const sp_grid *grid, int32_t n_arrays, const sp_array_desc *arrays,
                                 int32_t n_kernels, const sp_kernel *kernels, sp_comm *comm,
                                 stencil_program **out);
void stencil_program_destroy(stencil_program *prog);

sp_status stencil_program_layout(const stencil_program *prog, sp_layout *out);

/* Borrow dev_ptr (caller-owned, >= layout.bytes, 256-B aligned) as array `array`. */
sp_status stencil_program_bind(stencil_program *prog, int32_t array, void *dev_ptr);

/* Tuning/parity options; must precede fusion_plan_set / the first run.
 * Unknown keys or negative values: SP_E_ARG.  Results are bit-identical under
 * every option except "fmad"/"factor" (which select the perf build, R4/R17).
 *   "fmad"      0|1  FMA contraction in generated code (default 1; 0 = parity build)
 *   "factor"    0|1  perf build: terms sharing one multiplier summed first (default 1)
 *   "tile_x", "tile_y", "zchunk", "threads", "prefetch"   override the tile chooser
 *   "block_x", "block_y", "block_cby"   register block of a thread (0 = chooser)
 *   "zqueue"    0..2  z-reuse policy (see sp_tile_config.zqueue)
 *   "loader"    0 = TMA + mbarrier ring (default), 1 = cooperative loads
 *   "pdl"       0|1|2 programmatic dependent launch: off / fused groups / all
 *   "zwave"     S > 0: fused mode runs the z-wave schedule (sp_plan_wave_offsets)
 *   "zwave_streams" 1..8 waves in flight for "zwave" (default 2)
 *   "xpush"     1: peer-push halo exchange of TEMP epochs on several ranks (see
 *               sp_bind_peer); 0 (default): the communicator carries every epoch
 *   "regcap"    occupancy-aware register cap at JIT time (recompile with
 *               __maxnreg__ when a few registers cost a resident CTA, kept only
 *               without spills): 0 never, 1 peer-push kernels (default), 2 all
 *   "l2pf"      TMA L2 prefetch of input planes this many steps beyond the
 *               shared-memory ring (default 1; 0 off)
 *   "fastpath"  2: as 1, and the fast body also runs each chunk's warm-up steps (only
 *               chunks/tiles at the global boundary run the general body);
 *               1: a second, predicate-free copy of the step body for interior
 *               tiles/planes (fewer issued instructions, larger code); default 0
 *   "minblocks" __launch_bounds__ minimum resident CTAs (ptxas register budget)
 *   "rename"    1 (default): in run_fused on one rank of an undecomposed grid
 *               (nz_global == nz_local), every later group that stores a
 *               TEMP array stores into its own instance (a library-allocated buffer of
 *               the program layout; extra memory = sum over TEMPs of (writer groups - 1)
 *               arrays), so TEMP reuse creates no WAR/WAW ordering between groups.  The
 *               instances' ghost cells are copied from the bound TEMP buffer when it is
 *               (re)bound: rebind a TEMP after changing its ghost cells.  0: off
 *   "streams"   N (default 2): run_fused on one rank issues the launches along the group
 *               dependency DAG (sp_plan_dag) on up to N streams forked from and joined
 *               back into the caller's stream (events; graph-capturable); 1: in order
 *   "dagprio", "dagsched"   launch-DAG stream priority / assignment variants (measured off)
 *   "psleep"    ns: the TMA producer warp waits for a free ring slot with nanosleep
 *               back-off starting at this value (default 32; 0 = spin on try_wait)
 *   "phint", "pbar", "pow2ring"   measured-off producer-wait / ring experiments
 *   "frame"     1: region-vector evaluation of fused launches: every statement is
 *               evaluated on its whole extended region (tile + halo of complex
 *               fusion, §5.5.3) in 16-byte x-vectors of adjacent points
 *               enumerated linearly over the threads, instead of register blocks on
 *               the tile plus point-wise halo strips; launches with loop-bounded
 *               statements, peer push or clusters keep the block form; default 0.
 *               2: the same with ONE unit grid for all statements of a launch (the
 *               union of their regions; a statement skips units outside its own), so a
 *               unit's values at the unit's own position — centre and vertical taps — are
 *               kept in per-thread register queues instead of re-read from shared memory
 *   "cluster_x" 2..8: fused launches with a shared-memory stage extended in x run as
 *               thread-block clusters of that many x-neighbouring tiles; the x-halo
 *               columns a stage needs inside a neighbour's tile are read from that
 *               CTA's ring through distributed shared memory (remote mbarrier arrive
 *               + ld.shared::cluster) instead of recomputed (NEXT #2); launches whose
 *               tile columns do not divide by it stay unclustered; default 1 (off)
 *   "suspend_hint", "coef_const", "acc_split"   measured-off experiments
 *   "num_sms"   SM count assumed by the tile chooser (default 148)
 *   "l2_flush"  unused by the library (reserved) */
sp_status sp_program_set_option(stencil_program *prog, const char *key, int64_t value);

sp_status sp_program_counts(const stencil_program *prog, int32_t *n_stmts, int32_t *n_edges);
/* Copies up to cap edges (all RAW/WAR/WAW statement pairs in program order). */
sp_status sp_program_edges(const stencil_program *prog, int32_t cap, sp_edge *out, int32_t *n);

/* Kernel fission (§4.1, Algorithm 2; reading R8): connected
 * components of the graph joining each statement's output array with every
 * array it reads.  comp_of_stmt[i] receives the piece of statement i of the
 * kernel, pieces numbered in order of their first statement.  */
sp_status sp_fission_components(const stencil_program *prog, int32_t kernel, int32_t *comp_of_stmt,
                                int32_t *n_comp);

/* ---- plans ------------------------------------------------------------------
 * A plan is the new OEG: groups in execution order.  Group g
 * consists of members[group_begin[g] .. group_begin[g+1]) (statement refs;
 * listing every statement of a kernel fuses the whole kernel, listing a subset
 * is fission).  Checks: partition (every statement exactly once), order
 * (every dependency edge goes forward or stays inside a group), in-group
 * hazards (reading R11), resources (shared memory, deep-halo depth).  On error
 * the previous plan stays in place.  Host-side only: generates the kernels'
 * source; compilation happens in sp_compile or at the first run. */
sp_status fusion_plan_set(stencil_program *prog, int32_t n_groups, const int32_t *group_begin,
                          const sp_stmt_ref *members);

/* Greedy host-side plan search (the paper's search step, §3.2.4, with this
 * library's byte/flop/issue model as the objective): starts from fully fissioned
 * kernels (§4.1) and merges adjacent groups while the modelled time drops.
 * Writes at most cap groups: group_begin[cap+1], members[number of statements].
 * With group_begin == NULL only *n_groups is returned.  Does not set the plan. */
sp_status sp_plan_greedy(stencil_program *prog, int32_t cap, int32_t *n_groups,
                         int32_t *group_begin, sp_stmt_ref *members);
/* Launch configuration (0 = left to the model-driven chooser).  The thread
 * geometry must satisfy tile_x = (tile_x/block_x)*block_x and
 * tile_y = (threads/(tile_x/block_x)) * block_y * block_cby.
 * zqueue selects how values read at several planes are kept across z steps:
 * 0 = the program's "zqueue" option, 1 = shared-memory loads only, 2 = register
 * queues per statement, 3 = step-wide register queues of the input columns a
 * thread owns (results are bit-identical under every policy). */
typedef struct {
    int32_t tile_x, tile_y, zchunk, threads, prefetch, block_x, block_y, block_cby;
    int32_t zqueue;
    int32_t fastpath;  /* 0 = the program's "fastpath" option, 1 = off, 2 = on, 3 = on incl.
                          warm-up steps (this launch) */
    int32_t frame;     /* 0 = the program's "frame" option, 1 = off, 2 = on, 3 = on with
                          position-stable units and register z-reuse (this launch) */
} sp_tile_config;

/* Lazy-fission plan search (the paper's search step,
 * P:L140 §3.2.4 and §4.1).  Steps:
 *   1. metadata pre-step: the objective is evaluated for every original kernel and
 *      every fission piece (sp_fission_components) on its own ("lazy fission": the
 *      pieces' metadata is gathered first);
 *   2. exact DP over contiguous segmentations of the ORIGINAL kernels (no fission),
 *      segments of at most max_group_kernels kernels — the live-out set (R6) of a
 *      contiguous group depends on the group alone, so the DP optimum is exact;
 *   3. a grouping GA over fission pieces whose kernels start unfissioned (a
 *      kernel's pieces share one group until fission is applied to it): merge,
 *      split, move, group-injection crossover and the lazy-fission operator, which
 *      splits a kernel of a group that violates the shared-memory capacity;
 *      seeded with the DP optimum, the unfused plan and sp_plan_greedy's plan.
 *      Fitness is the paper's dynamic penalty
 *          f_p(x) = f(x) + sum_i C_i delta_i - C_SM delta_SM
 *      with f = sum of the groups' times (a violating group is charged its units'
 *      pre-step times), delta_i = cyclic group order / in-group hazard (R11, R2') /
 *      no tile fits (resources), C_SM = +c_sm when a kernel of the smem-violating
 *      group can still be fissioned (the relaxation fission offers) and -c_sm when
 *      not.  Independent statements may be grouped out of program order.
 * Objective 0: this library's launch-time model (host only, deterministic for the
 * options).  Objective 1: measured — every candidate group is JIT-compiled and timed
 * on the current device with CUDA events on `stream` (median of `reps` launches,
 * L2 flushed before each; the paper's empirical metadata, §3.2.1); the
 * program's arrays must be bound, and their contents are overwritten.
 * With candidate configurations (measured objective) every group is also timed at
 * each one that fits and costs its fastest; `configs` (nullable, >= cap entries,
 * written with the groups) receives each returned group's configuration for
 * sp_plan_tune (all zero: the chooser's).  Output as sp_plan_greedy; `report`
 * (nullable) receives costs and counts.  Does not set the plan.  Errors: SP_E_ARG
 * (options), SP_E_STATE (measured: an array not bound), SP_E_JIT / SP_E_CUDA
 * (measured: compilation or a kernel failed). */
typedef struct {
    int32_t generations;        /* GA generations (0: pre-step + DP + seeds only)            */
    int32_t population;         /* GA population (clamped to >= 4)                            */
    uint64_t seed;              /* GA random stream                                           */
    int32_t objective;          /* 0 = launch-time model (host), 1 = measured on the device   */
    int32_t max_group_kernels;  /* DP segment bound in original kernels (0 -> 8)              */
    int32_t reps;               /* measured: timed launches per group, median (0 -> 5)        */
    double c_violation;         /* C_i per violated constraint, x the unfused plan cost (0 -> 1) */
    double c_sm;                /* |C_SM|, x the unfused plan cost (0 -> 0.5)                  */
    int32_t n_configs;          /* measured: candidate tile configurations timed per group    */
    const sp_tile_config *configs; /* besides the chooser's; a group costs its fastest one    */
} sp_search_options;
typedef struct {
    double cost_us;             /* objective of the returned plan                             */
    double dp_cost_us;          /* best contiguous unfissioned plan (step 2)                  */
    double unfused_cost_us;     /* one group per original kernel                              */
    int32_t groups_evaluated;   /* distinct groups the objective evaluated                    */
    int32_t fissioned_kernels;  /* kernels whose pieces the returned plan separates           */
    int32_t generations_run;
} sp_search_report;
sp_status sp_plan_search_ex(stencil_program *prog, const sp_search_options *opts, sp_stream stream,
                            int32_t cap, int32_t *n_groups, int32_t *group_begin, sp_stmt_ref *members,
                            sp_tile_config *configs, sp_search_report *report);
/* sp_plan_search_ex with the model objective and default constants.  Host-only. */
sp_status sp_plan_search(stencil_program *prog, int32_t generations, int32_t population, uint64_t seed,
                         int32_t cap, int32_t *n_groups, int32_t *group_begin, sp_stmt_ref *members);

/* mode 0 = unfused (one launch per original kernel), 1 = fused plan. */
sp_status sp_plan_count(const stencil_program *prog, int32_t mode, int32_t *n_launches);
sp_status sp_plan_report(const stencil_program *prog, int32_t mode, int32_t launch,
                         sp_group_report *out);
sp_status fusion_plan_report(const stencil_program *prog, int32_t group, sp_group_report *out);
/* Generated CUDA source of a mode (for inspection); *len receives the full size. */
sp_status sp_plan_source(stencil_program *prog, int32_t mode, char *buf, size_t cap, size_t *len);

/* Empirical tuning hook (the paper's per-kernel block-size tuning, §4.2):
 * pin the configuration of one launch of a mode; cfg == NULL removes the pin.
 * Re-analyses and regenerates the mode (JIT at the next compile/run).  Pins of
 * the fused mode are dropped when a new plan is set.  SP_E_RESOURCES if the
 * configuration does not fit. */
sp_status sp_plan_tune(stencil_program *prog, int32_t mode, int32_t launch, const sp_tile_config *cfg);

/* Halo-exchange schedule of one launch on several ranks: the
 * arrays whose ghost planes are received right before it (up to cap written to
 * arrays[], *n = total), with the planes received into the bottom ghost
 * (below[i]) and the top ghost (above[i]); below/above may be NULL.  An array
 * is received once per epoch (step start, or a launch that stores it, up to the
 * next), at the largest depth any reader of the epoch needs (each <= zhalo):
 * an epoch that begins at a store before its first launch that reads the array
 * beyond the slab, every step-start epoch in one exchange before the step's
 * first launch.  With option "xpush" the epochs of TEMP arrays that begin at a
 * store are pushed by the storing kernel instead and do not appear here.
 * run_unfused / run_fused perform exactly this exchange, overlapped with the
 * launch's interior planes; host-only (no GPU needed). */
sp_status sp_plan_exchange(stencil_program *prog, int32_t mode, int32_t launch, int32_t cap,
                           int32_t *arrays, int32_t *below, int32_t *above, int32_t *n);
/* z-wave schedule of the fused mode (options "zwave" = S planes per wave,
 * "zwave_streams" = waves in flight on that many streams; single rank only).
 * In wave w, launch i evaluates output planes [w*S - off_i, (w+1)*S - off_i)
 * of the slab; the skew off_i >= 0 is the smallest that keeps every plane a
 * launch reads or writes disjoint from the planes of concurrently running or
 * later-issued waves of other launches (RAW: off_i >= off_j + z-reach above,
 * WAR: off_i >= off_j + z-reach below, WAW: off_i >= off_j for j < i), so
 * results are bit-identical to plan order.  Writes up to cap offsets, *n = the
 * number of fused launches.  Host-only (no GPU needed). */
sp_status sp_plan_wave_offsets(stencil_program *prog, int32_t cap, int32_t *off, int32_t *n);
/* JIT-compile (NVRTC, sm_100a) without launching; needs no GPU. */
sp_status sp_compile(stencil_program *prog, int32_t mode);
/* Compile if needed and load the mode's modules on the current device (needs a
 * GPU).  run_* load lazily; call this first when ranks are driven from several
 * threads of one process (loopback), since a module load may synchronise the
 * device while a neighbour's kernels wait for this rank. */
sp_status sp_load(stencil_program *prog, int32_t mode);

/* ---- execution ---------------------------------------------------------- */
/* Every original kernel once, in program order: one launch per kernel, each
 * reading its inputs from and writing all its outputs to HBM. */
sp_status run_unfused(stencil_program *prog, sp_stream stream);
/* The current plan's groups in order (SP_E_STATE if no plan).  On several
 * ranks a group whose schedule (sp_plan_exchange) receives ghost planes runs
 * its interior planes while the exchange is in flight on the communicator's
 * stream, then its boundary planes. */
sp_status run_fused(stencil_program *prog, sp_stream stream);
/* One launch of a mode (profiling / per-kernel timing); no exchange. */
sp_status sp_run_launch(stencil_program *prog, int32_t mode, int32_t launch, sp_stream stream);
/* Number of kernel launches one run_unfused (mode 0) / run_fused (mode 1) call
 * issues with the current communicator and options: one per live launch; on
 * several ranks a launch that receives ghost planes first (sp_plan_exchange) is
 * an interior launch plus one boundary launch covering both slab ends (one
 * launch when its interior is empty); under "zwave" one per non-empty wave of
 * each launch.  NCCL's own kernels are not counted.  Host-only. */
sp_status sp_run_launch_count(stencil_program *prog, int32_t mode, int32_t *n);

/* Launch DAG of run_fused (mode 1) with options "rename" / "streams" (one rank): the
 * earlier launches launch `launch` depends on — RAW / WAR / WAW on the buffer instance
 * of an array (with "rename" every later writer group of a TEMP stores into its own
 * instance, so TEMP reuse adds no WAR/WAW edge) — written to deps[0..min(cap, n)) with
 * *n_deps = n, and the stream index it is issued on (0 = the caller's stream).  Without
 * those options every launch depends on its predecessors through the arrays alone, and
 * all run on stream 0.  Host-only; also valid for mode 0 (stream 0, plain edges). */
sp_status sp_plan_dag(stencil_program *prog, int32_t mode, int32_t launch, int32_t cap, int32_t *deps,
                      int32_t *n_deps, int32_t *stream);

/* Exchange `depth` ghost planes of each listed array with the z-neighbours
 * (ncclSend/ncclRecv grouped; planes are contiguous, no packing).  Requires
 * a communicator; 1 <= depth <= zhalo. */
sp_status exchange_halos(stencil_program *prog, int32_t n, const int32_t *arrays, int32_t depth,
                         sp_stream stream);

const char *sp_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* STENCILFUSE_H */
