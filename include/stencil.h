/*
 * include/stencil.h -- C ABI of the B200-native StencilMART hot path.
 *
 * StencilMART (Sun et al., IPDPS'22; /root/reference/PAPER.md, cited "P:L<line>")
 * profiles every stencil under every optimization combination (OC) to label
 * the best one: "the performance of each stencil input is profiled with
 * different OCs on the target GPU, and the OC with the best performance is
 * labeled. Specifically, the StencilMART randomly searches the parameter
 * settings under each OC and selects the shortest execution time" (P:L119,
 * §IV-A; also P:L234, §V-A.2). This library is that data-parallel path: the
 * sweep of one arbitrary 2-D/3-D stencil under any OC of Table I, and the
 * per-OC timing sweep that produces the label.
 *
 * Conventions shared by every entry point
 * ---------------------------------------
 * - Every function returns a stencil_status_t (0 = OK, < 0 = error) unless
 *   stated otherwise; the thread-local message of the last error is returned by
 *   stencil_last_error().
 * - Grids are dense, row-major, slowest dimension first: 3-D [nz][ny][nx],
 *   2-D [ny][nx] (x contiguous), element type per stencil_dtype_t.
 * - Device pointers are owned by the caller (PyTorch in the Python binding),
 *   must be at least 16-byte aligned and hold the whole grid. Host pointers
 *   (stencil_run_host) are plain caller memory.
 * - Argument validation happens before any CUDA call, so invalid arguments are
 *   reported as STENCIL_E_INVAL / STENCIL_E_OC_INVALID even without a GPU.
 * - Work is enqueued on the plan's stream (stencil_plan_set_stream; default:
 *   the legacy default stream) and is asynchronous w.r.t. the host unless
 *   stated otherwise. CUDA errors are reported by the call that detects them.
 * - A plan must not be used concurrently from several host threads; distinct
 *   plans are independent.
 */
#ifndef STENCILMART_STENCIL_H
#define STENCILMART_STENCIL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define STENCIL_ABI_VERSION 2

/* Opaque plan: one stencil on one grid shape under one OC and parameter
 * setting. Created by stencil_plan_create, owned by the caller, released by
 * stencil_plan_destroy. It owns its compiled kernels, TMA descriptors, events
 * and (multi-GPU) its NCCL communicator. */
typedef struct stencil_plan_s *stencil_plan_t;

typedef enum { STENCIL_F32 = 0, STENCIL_F64 = 1 } stencil_dtype_t;

/* OC bitmask (Table I). OC id = OR of these bits; 0 is the
 * plain kernel ("each GPU thread works on a single output point").
 * Table I constraints: BM and CM are mutually exclusive; RT and PR are only
 * valid with ST. Exactly 30 ids are valid (6 without ST, 24 with ST). */
enum {
    STENCIL_OC_ST = 1,   /* streaming (2.5-D blocking, concurrent streaming) */
    STENCIL_OC_BM = 2,   /* block merging: k adjacent outputs per thread */
    STENCIL_OC_CM = 4,   /* cyclic merging: k outputs a fixed distance apart */
    STENCIL_OC_RT = 8,   /* retiming: per-plane partial sums */
    STENCIL_OC_PR = 16,  /* prefetching: next plane loaded during compute */
    STENCIL_OC_TB = 32   /* temporal blocking: T fused time steps */
};
#define STENCIL_NUM_OC 30

typedef enum {
    STENCIL_OK = 0,
    STENCIL_E_INVAL = -1,          /* bad argument (dims, order, access, coeffs, dtype, pointers) */
    STENCIL_E_OC_INVALID = -2,     /* OC violates Table I */
    STENCIL_E_OC_INFEASIBLE = -3,  /* OC + setting exceeds a hardware limit (the paper's OC "crash") */
    STENCIL_E_NOMEM = -4,
    STENCIL_E_CUDA = -5,
    STENCIL_E_NCCL = -6,
    STENCIL_E_NVRTC = -7,          /* kernel specialisation failed */
    STENCIL_E_STATE = -8           /* call not valid in the plan's current state (e.g. no workspace) */
} stencil_status_t;

/* Parameter setting of an OC (§IV-E: numeric parameters are powers of
 * two, Boolean parameters are {0,1}, enumerations start at 1). A field equal to
 * 0 (-1 for smem) selects the library default for the OC and dtype; fields an
 * OC does not use are ignored. */
typedef struct {
    int32_t smem;         /* Boolean "shared memory usage"; OCs base/BM/CM only:
                             1 = stage an (x,y,z) tile + halo in shared memory, 0 = global loads */
    int32_t bx;           /* CTA tile width along x in outputs (power of two, 8..256) */
    int32_t by;           /* threads per CTA along y (power of two) */
    int32_t bz;           /* non-streaming tiled kernels: output planes per CTA */
    int32_t vx;           /* outputs per thread along x (1, 2, 4): one 128-bit vector */
    int32_t merge;        /* BM/CM merge factor k (1..8): outputs per thread along y; in 2-D
                             streaming OCs (planes are single rows) along x -- BM adjacent
                             vectors, CM vectors bx/k columns apart */
    int32_t stream_chunk; /* ST: output planes per CTA ("concurrent streaming") */
    int32_t tb_steps;     /* TB: time steps fused per launch (2..8) */
    int32_t pr_stages;    /* PR: planes in flight in the TMA pipeline (1..8; the settings
                             sampler draws the enumeration 2..4; 1 = no prefetching) */
    int32_t reserved[3];  /* must be 0 */
} stencil_params_t;

/* Read-only facts about a plan (for tests, reports and the sweep). */
typedef struct {
    int32_t ndim, order, nnz, dtype;
    int32_t ext[6];           /* z_lo, z_hi, y_lo, y_hi, x_lo, x_hi: neighbour extents (<= order) */
    uint32_t oc;
    stencil_params_t params;  /* the resolved setting (defaults filled in) */
    int32_t kernel_family;    /* 0 naive, 1 tiled, 2 stream, 3 stream+TB */
    int32_t smem_bytes;       /* dynamic shared memory per CTA */
    int32_t threads;          /* threads per CTA */
    int32_t regs;             /* registers per thread of the main kernel (0 until compiled) */
    int32_t uses_tma;         /* 1 if halo tiles are staged with cp.async.bulk.tensor; 0 =
                                 element-wise cp.async (rows that are not 16-byte multiples,
                                 boxes wider than 256) or global loads (naive) */
    int64_t points;           /* interior points updated per time step (global grid) */
    char kernel_name[128];    /* lowered name of the main kernel */
    int32_t reg_split[2];     /* warp-specialised ST_TB_RT kernel: registers per thread of the
                                 producer/intermediate-stage warps and of the last-stage warps
                                 after setmaxnreg (0, 0 = no split) */
    int32_t xshift;           /* ST_TB_RT kernel uses the aligned-window ring geometry (§6.1) */
    int32_t host_chunks;      /* z-chunks of the last stencil_run_host (0 = not pipelined) */
} stencil_plan_info_t;

/* ---------------------------------------------------------------------------
 * Plan lifetime
 * ------------------------------------------------------------------------- */

/* Create a plan (§8(a) rows a1-a3 of SURVEY.md).
 *   ndim    2 or 3.
 *   dims    ndim extents, slowest first ([nz,ny,nx] or [ny,nx]); each >= 2*order+1.
 *           With a communicator set later, dims[0] is the LOCAL slab depth.
 *   order   r in 1..4: frame width and access-tensor radius (order = maximum
 *           extent of the neighbours).
 *   access  uint8[(2r+1)^ndim], row-major [dz+r][dy+r][dx+r]; 1 = accessed.
 *           The centre must be 1; the maximum extent may be < r.
 *   coeffs  double[(2r+1)^ndim], same layout; must be 0 where access == 0.
 *           Rounded to the plan dtype once, round-to-nearest-even.
 *   dtype   STENCIL_F32 or STENCIL_F64 (arithmetic type of the sweep).
 *   oc      OC bitmask; STENCIL_E_OC_INVALID if it violates Table I.
 *   params  NULL = defaults.
 * The update computed by every OC is
 *   u_{t+1}[p] = sum_{o in S} c_o u_t[p+o]   for r <= p_k < n_k - r on every axis,
 *   u_{t+1}[p] = u_t[p]                     elsewhere (the frame; C-1),
 * each sum evaluated as one fused-multiply-add chain in lexicographic
 * (dz,dy,dx) order, so every OC returns bitwise the same grid.
 * Kernel specialisation (NVRTC, sm_100a) happens here; the result is cached
 * per process and, if STENCIL_CACHE_DIR (default ~/.cache/stencilmart) is
 * writable, on disk. Needs a CUDA device for the compile+load step unless the
 * environment variable STENCIL_DEFER_COMPILE=1 is set (compile at first run). */
int stencil_plan_create(stencil_plan_t *plan, int ndim, const int64_t *dims, int order,
                        const uint8_t *access, const double *coeffs, stencil_dtype_t dtype,
                        uint32_t oc, const stencil_params_t *params);

/* Release the plan and everything it owns. NULL is a no-op. */
void stencil_plan_destroy(stencil_plan_t plan);

/* Stream on which stencil_run / stencil_oc_sweep enqueue work (a cudaStream_t). */
int stencil_plan_set_stream(stencil_plan_t plan, void *cuda_stream);

/* Bytes of device workspace stencil_run needs for steps >= 2 (one grid). */
size_t stencil_plan_workspace_bytes(stencil_plan_t plan);

/* Caller-owned device workspace (>= stencil_plan_workspace_bytes, 16-B aligned).
 * Must stay valid while the plan runs. */
int stencil_plan_set_workspace(stencil_plan_t plan, void *dev_ptr, size_t bytes);

/* Fill *info. Host-only. */
int stencil_plan_info(stencil_plan_t plan, stencil_plan_info_t *info);

/* ---------------------------------------------------------------------------
 * Sweeps
 * ------------------------------------------------------------------------- */

/* Advance `steps` (>= 0) time steps: out = S^steps(in). `in` is preserved;
 * in != out (STENCIL_E_INVAL otherwise); steps == 0 copies. steps >= 2 needs a
 * workspace. The frame of `in` is copied once into out (and the workspace);
 * TB OCs launch ceil(steps/T) times, the last launch fusing the remainder. */
int stencil_run(stencil_plan_t plan, const void *in_dev, void *out_dev, int steps);

/* End-to-end form: `in_host` / `out_host` are host buffers of the grid (pinned
 * memory for full PCIe speed). The call copies in_host to device buffers it
 * owns, runs `steps` steps with the plan's OC, copies the result back and
 * returns when out_host holds it (the plan's stream is synchronised). Single-GPU
 * plans whose slowest view axis has >= 64 planes and whose grid holds >= 32 MiB
 * are pipelined over z-chunks:
 * the upload of chunk k+1, a time-skewed sweep of chunk k and the download of
 * chunk k-1 overlap on two internal copy streams; the result is bitwise that of
 * stencil_run. Errors as stencil_run. */
int stencil_run_host(stencil_plan_t plan, const void *in_host, void *out_host, int steps);

/* The label generator: for each of the 30 OCs in ascending id
 * order and each of `settings_per_oc` parameter settings (the plan's own
 * setting's defaults first, then seeded random powers of two, see
 * stencil_sample_params), create a plan for the same stencil, run one warm-up,
 * then `reps` timed runs of `steps` steps with CUDA events on the plan's
 * stream; the setting's time is the median, the OC's time the minimum over its
 * settings. Infeasible OCs get +INF. best_oc = argmin over finite times, ties
 * to the smallest id. With a communicator, per-OC times are the max over ranks
 * (all ranks return identical vectors). `in` is preserved, `out` receives the
 * last run's result. Error containment: a setting whose plan is infeasible
 * (E_OC_INFEASIBLE) or whose launch fails while the CUDA context stays usable
 * counts as a crash of that setting (+INF, the row's status says why) and the
 * sweep goes on; E_INVAL from a sampled setting (a sampler bug), a sticky CUDA
 * error, an NCCL error or an NVRTC failure fails the whole call. Outputs:
 *   times_ms[30], oc_ids[30] (ascending), best_params[30], *best_oc.
 * Synchronises the plan's stream. */
int stencil_oc_sweep(stencil_plan_t plan, const void *in_dev, void *out_dev, int steps,
                     int settings_per_oc, int reps, uint64_t seed,
                     float *times_ms, uint32_t *oc_ids, stencil_params_t *best_params,
                     uint32_t *best_oc);

/* ---------------------------------------------------------------------------
 * OC lattice and parameter space (host only, no GPU needed)
 * ------------------------------------------------------------------------- */

/* 1 if `oc` satisfies Table I, else 0. */
int stencil_oc_valid(uint32_t oc);

/* Write the 30 valid OC ids in ascending order into ids[30]; returns 30. */
int stencil_oc_list(uint32_t *ids);

/* Static name of an OC ("base", "ST", "TB_CM", "ST_BM_RT_PR", ...: components in
 * the order ST, TB, BM, CM, RT, PR); NULL for an invalid id. */
const char *stencil_oc_name(uint32_t oc);

/* The k-th (k >= 0) sampled setting for `oc` under `seed`: k = 0 is the
 * default setting, k >= 1 draws each numeric field as a power of two from the
 * OC's range with a counter-based hash of (seed, oc, k). Deterministic. */
int stencil_sample_params(uint32_t oc, int ndim, stencil_dtype_t dtype, uint64_t seed, int k,
                          stencil_params_t *out);

/* ---------------------------------------------------------------------------
 * Stencil representation (§IV-C; host only)
 * ------------------------------------------------------------------------- */

/* Table II feature set: order = maximum (Chebyshev) extent of the
 * non-zeros, nnz, sparsity = nnz / 9^ndim (the fixed (2*4+1)^d tensor of
 * P:L135), nnz_order[n-1] = non-zeros in ring n, nnz_ratio[n-1] =
 * nnz_order[n-1] / |ring n| (|ring n| = (2n+1)^d - (2n-1)^d). */
typedef struct {
    int32_t order;
    int32_t nnz;
    double sparsity;
    int32_t nnz_order[4];
    double nnz_ratio[4];
} stencil_features_t;

int stencil_features(int ndim, int order, const uint8_t *access, stencil_features_t *out);

/* The access tensor embedded, centred, in the fixed 9^ndim binary tensor of
 * Fig. 6 (the ConvNet / ConvMLP input). out9: 729 (3-D) or 81 bytes. */
int stencil_embed_tensor(int ndim, int order, const uint8_t *access, uint8_t *out9);

/* Rows of the last stencil_oc_sweep on `plan` (the paper's stencil dataset:
 * "each parameter setting and its corresponding execution time are also
 * stored"): one row per (OC, setting) tried, in sweep order. Writes at
 * most max_rows rows and the total count to *nrows. time_ms = +INF if the
 * setting did not run; `status` says why: STENCIL_OK (timed),
 * STENCIL_E_OC_INFEASIBLE (a resource limit: the paper's "crash"), or
 * the code of a launch error that left the CUDA context usable (contained to
 * this setting; see stencil_oc_sweep). */
typedef struct {
    uint32_t oc;
    int32_t setting;          /* k of stencil_sample_params */
    stencil_params_t params;  /* resolved setting (defaults filled in; the raw
                                 sample when the plan could not be created) */
    float time_ms;            /* median of the timed runs */
    int32_t status;           /* STENCIL_OK or the reason time_ms is +INF */
} stencil_sweep_row_t;

int stencil_sweep_rows(stencil_plan_t plan, stencil_sweep_row_t *rows, int max_rows, int *nrows);

/* ---------------------------------------------------------------------------
 * OC analysis over a stencil dataset (§III-A..C, §IV-D, §V-A.2;
 * SURVEY NEXT-4; host only, no CUDA call)
 * ------------------------------------------------------------------------- */

/* times: [n_stencils][n_oc] row-major host array of per-OC shortest times
 * (ms; a value that is not finite and > 0 = the OC did not run on that
 * stencil). 1 <= n_oc <= 64, n_classes >= 1. Every output is optional
 * (NULL = not wanted), host memory owned by the caller:
 *   gap[n_stencils]   worst / best time per stencil (Fig. 1); NaN if no OC ran;
 *   wins[n_oc]        stencils each OC is best for (Fig. 2; ties -> smaller column);
 *   pcc[n_oc*n_oc]    Pearson correlation between OC columns of the per-stencil
 *                     performance t_best/t, over the stencils where both ran
 *                     (Fig. 3); < 3 common stencils or zero variance -> 0;
 *   group[n_oc]       class of each OC after merging pairs by |PCC| descending
 *                     (ties -> smaller (a,b)) until n_classes groups remain
 *                     ("reduce the number of predicted
 *                     OCs to 5"); groups numbered by their smallest member;
 *   rep[n_classes]    the member with the most wins ("the OC that obtains
 *                     the best performance under more cases"; ties -> smaller
 *                     column); -1 for unused classes when n_oc < n_classes;
 *   labels[n_stencils] class of each stencil = group of its best OC, -1 if none ran.
 * Errors: E_INVAL on bad sizes or a null `times` with n_stencils > 0. */
int stencil_oc_analysis(int n_stencils, int n_oc, const double *times, int n_classes, double *gap,
                        int32_t *wins, double *pcc, int32_t *group, int32_t *rep, int32_t *labels);

/* ---------------------------------------------------------------------------
 * Synthetic inputs (the counter-based generator of DESIGN.md, reading C-3)
 * ------------------------------------------------------------------------- */

/* FMA-throughput probe (measurement only): enqueue on
 * `cuda_stream` one launch of blocks_per_sm (1..8) x SM-count CTAs of 256
 * threads, each thread running 8 independent fused-multiply-add chains for
 * iters x 8 steps in `dtype`; *flops receives the launch's floating-point
 * operations (2 per FMA). The caller times the launch (CUDA events on the same
 * stream) to get the measured FMA peak that the "alu" roofline of FMA-bound
 * stencils divides by -- the paper lists each GPU's FP64 peak.
 * `sink` is a device buffer of at least one element of `dtype` (written only in
 * a case that never happens; it keeps the chains live). E_INVAL on bad
 * arguments. */
int stencil_fma_probe(stencil_dtype_t dtype, int64_t iters, int blocks_per_sm, void *sink, void *cuda_stream,
                      double *flops);

/* Fill a device box of shape box_dims (ndim values, slowest first) whose
 * element i holds value(h(seed, g)), g = the row-major linear index of
 * (origin + i) in a grid of shape global_dims. kind 0 = uniform in [1,2),
 * kind 1 = integers in [-1023, 1023]. Enqueued on `cuda_stream`. */
int stencil_fill_field(void *dev_ptr, stencil_dtype_t dtype, int ndim, const int64_t *box_dims,
                       const int64_t *origin, const int64_t *global_dims, uint64_t seed, int kind,
                       void *cuda_stream);

/* ---------------------------------------------------------------------------
 * Multi-GPU (one process per GPU; grids slab-decomposed along dims[0])
 * ------------------------------------------------------------------------- */

/* Fill id[128] with a fresh NCCL unique id (call on rank 0, broadcast it). */
int stencil_nccl_unique_id(uint8_t *id);

/* Attach the plan (3-D only) to a communicator of `nranks` ranks. The plan's
 * grid becomes rank `rank`'s slab of a global grid whose depth is the sum of
 * the ranks' dims[0] (ranks ordered along z); the frame exists only at the
 * global z faces. Device buffers passed to stencil_run (and the workspace)
 * then hold dims[0] + 2G planes: G ghost planes, the dims[0] owned planes,
 * G ghost planes (G = stencil_plan_ghost_planes(plan) = 4*order; dims[0] must
 * be >= 2G). Each launch computes the edge planes first, exchanges the halo
 * planes with ranks +-1 (ncclSend/ncclRecv on a comm stream: T*extent planes
 * every T fused steps) and computes the interior meanwhile; at the start of
 * stencil_run the ghost planes of `in` are overwritten with the neighbours'
 * owned planes. Collective: all ranks call it with the same id; tb_steps <= 4. */
int stencil_plan_set_comm(stencil_plan_t plan, const uint8_t *id, int rank, int nranks);

/* Same as stencil_plan_set_comm, but adopting an existing NCCL communicator
 * (an ncclComm_t, e.g. the one torch.distributed's NCCL process group owns);
 * the plan does not destroy it. The communicator must span `nranks` ranks with
 * this process at `rank`, on the current device, and outlive the plan. */
int stencil_plan_set_nccl_comm(stencil_plan_t plan, void *nccl_comm, int rank, int nranks);

/* Attach `plan` to the communicator of `src` (set by either call above; a
 * unique id initialises only one communicator). `src` must outlive `plan`. */
int stencil_plan_share_comm(stencil_plan_t plan, stencil_plan_t src);

/* Single-device test form of the decomposition: link `nranks` plans of one
 * process (rank k = plans[k], same stencil/OC/dtype/plane shape) as slabs of one
 * global grid; halos move by cudaMemcpyAsync between their buffers, with the
 * same schedule as the NCCL path. Run them with stencil_run_group. */
int stencil_plans_link_loopback(stencil_plan_t *plans, int nranks);

/* Advance a loopback group (or one plan: nplans = 1) by `steps` steps:
 * ins[k] -> outs[k] for every slab k. Same semantics as stencil_run. */
int stencil_run_group(stencil_plan_t *plans, int nplans, const void *const *ins, void *const *outs,
                      int steps);

/* Fused device-initiated halo (not in the paper): the "P2P"
 * transport. Instead of NCCL send/recv after the edge kernels, the edge
 * kernels themselves store each output plane that a neighbour needs into that
 * neighbour's ghost planes through peer memory (NVLink P2P stores issued tile
 * by tile with the local stores), then a one-thread kernel publishes an epoch
 * with a system-scope release store into the neighbour's flag word; before its
 * next edge kernels a rank waits (acquire loads) until both neighbours have
 * published that epoch. No NCCL kernel, no comm stream, no staging copy.
 *   self  this rank's registered grids: stencil_run(plan, in, out, ...) must be
 *         called with in == self->in, out == self->out and the workspace set to
 *         self->ws (the neighbours write into their ghost planes);
 *   lo/hi rank-1 / rank+1 (NULL at the global faces): their registered grids
 *         and flag words, mapped into this process (stencil_ipc_open_handle, or
 *         plain pointers for plans of one process);
 *   flags 16 bytes of device memory per rank (flags[0] is written by rank-1,
 *         flags[1] by rank+1, flags[2] is the rank's own epoch counter, kept
 *         on the device), zeroed by the caller before any rank registers; one
 *         flag buffer serves every plan of the rank (epochs are counted per
 *         flag buffer, so all ranks must run the same sequence of runs; a new,
 *         zeroed buffer starts a new count);
 *   owned_planes  the rank's dims[0].
 * Slab layout, ghost depth and edge/interior split as stencil_plan_set_comm.
 * Registration also compiles and loads every kernel a run can launch (the main
 * one and the TB remainder kernels), so that no module load happens once ranks
 * sharing a device wait on each other's flags.
 * stencil_oc_sweep needs an NCCL communicator (E_STATE with this transport). */
typedef struct {
    void *in, *out, *ws;
    uint32_t *flags;
    int64_t owned_planes;
} stencil_p2p_buffers_t;

int stencil_plan_set_p2p(stencil_plan_t plan, int rank, int nranks, const stencil_p2p_buffers_t *self,
                         const stencil_p2p_buffers_t *lo, const stencil_p2p_buffers_t *hi);

/* CUDA IPC for the P2P transport (one process per GPU): the handle of the
 * allocation that contains dev_ptr (64 bytes) and dev_ptr's byte offset in it;
 * open maps a peer's allocation into this process and returns the address of
 * the same byte (base + offset); close unmaps it (pass what open returned and
 * the same offset). */
int stencil_ipc_get_handle(const void *dev_ptr, uint8_t *handle, int64_t *offset);
int stencil_ipc_open_handle(const uint8_t *handle, int64_t offset, void **dev_ptr);
int stencil_ipc_close(void *dev_ptr, int64_t offset);

/* G, the ghost planes on each side of the plan's slab (0 without a communicator). */
int stencil_plan_ghost_planes(stencil_plan_t plan);

/* Host-only halo layout of one exchange (for tests and tools): for a slab of n
 * owned planes stored at [G, G+n) whose stencil reaches zlo_g planes below and
 * zhi_g above, writes out[8] = {recv_lo_begin, recv_lo_count, send_lo_begin,
 * send_lo_count, send_hi_begin, send_hi_count, recv_hi_begin, recv_hi_count}
 * in local plane indices (lo = rank-1, hi = rank+1; counts 0 at global faces). */
int stencil_slab_halo(int ghost, int64_t n, int zlo_g, int zhi_g, int rank, int nranks, int64_t *out);

/* Slab layout of `rank` among `nranks` for a global depth nz_global: writes
 * {z_begin, z_end} of the rank's slab (near-equal split). Host only. */
int stencil_slab_range(int64_t nz_global, int rank, int nranks, int64_t *z_begin, int64_t *z_end);

/* ---------------------------------------------------------------------------
 * Diagnostics
 * ------------------------------------------------------------------------- */

/* Thread-local message of the last error (empty string if none). */
const char *stencil_last_error(void);

/* Kernel timing: with enable = 1, stencil_run brackets every sweep-kernel
 * launch with CUDA events on the plan's stream; stencil_plan_kernel_time then
 * synchronises the last event and returns (and resets) the summed device time
 * of those launches and their count. Used by the benchmark's roofline figure
 * (achieved bytes / average launch duration). */
int stencil_plan_set_timing(stencil_plan_t plan, int enable);
int stencil_plan_kernel_time(stencil_plan_t plan, double *kernel_ms, int64_t *launches);

/* Number of kernels this library launched in this process so far (for the
 * benchmark's gpu_launches count). */
uint64_t stencil_launch_count(void);

/* STENCIL_ABI_VERSION of the loaded library. */
int stencil_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* STENCILMART_STENCIL_H */
