/*
 * orion.h -- the C ABI of liborion, the B200-native (sm_100a) occupancy-tuned hot
 * path of "Orion: A Framework for GPU Occupancy Tuning" (Hayes et al., Middleware'16).
 *
 * Citations: P:L<n> = PAPER.md line n (section / figure / equation given beside it).
 * The boundary follows the paper's two questions (§3, P:L133-P:L137 and P:L175):
 *   (1) "how to generate the code given any occupancy level"
 *         -> orion_levels + orion_build_variants (+ orion_launch to realise a level);
 *   (2) "how to choose the best code version out of all the code versions"
 *         -> orion_tuner_create + orion_tune_step (two-level selection, Fig. 3).
 *
 * Conventions (every function):
 *   - Returns orion_status: ORION_OK (0) or a negative error code.  Errors are never
 *     fatal; orion_last_error() returns a thread-local message (driver string, ptxas log).
 *   - Ownership: the CALLER owns all image / grid buffers (device pointers, e.g. torch
 *     tensors' data_ptr()) and the CUDA stream (a CUstream / cudaStream_t passed as
 *     void*; NULL = the legacy default stream).  The LIBRARY owns compiled cubins,
 *     CUmodules, CUDA events and tuner state; each has a create/destroy pair.
 *   - No device allocation happens inside orion_launch / orion_tune_step.
 *   - Handles are not thread-safe: use one per stream / rank.
 *   - Every device entry point uses the CUDA primary context of the given device (the
 *     same context PyTorch uses); host-only entry points never touch the GPU.
 *   - Image layout: float4 RGBA (x,y,z,w = r,g,b,a) in [0,1], row-major, pitch = width
 *     pixels; stencil grids: float32, row-major, pitch = width.
 */
#ifndef ORION_H
#define ORION_H

#ifdef __cplusplus
extern "C" {
#endif

typedef int orion_status;
enum {
    ORION_OK = 0,
    ORION_E_INVALID = -1,             /* bad argument (NULL, out-of-range, unknown kernel id)      */
    ORION_E_CAPACITY = -2,            /* output array too small; *n_out holds the size needed      */
    ORION_E_INFEASIBLE = -3,          /* requested occupancy level cannot be realised               */
    ORION_E_COMPILE = -4,             /* ptxas (nvPTXCompiler) failed; log in orion_last_error()   */
    ORION_E_CUDA = -5,                /* CUDA driver error (or no driver / no GPU)                  */
    ORION_E_OCCUPANCY_MISMATCH = -6,  /* realised CTAs/SM (driver occupancy API) != the level's k   */
    ORION_E_STATE = -7                /* call not valid in the object's current state               */
};

/* Limiter bits of orion_level.limiter (which limits equal the realised CTA count). */
enum { ORION_LIM_REGS = 1, ORION_LIM_SMEM = 2, ORION_LIM_WARPS = 4, ORION_LIM_BLOCKS = 8 };

/* Device resource limits -- the inputs of Eq. (1) (P:L121-P:L127: Nreg, Nsmem, Smax) plus
 * the allocation granularities the "NVIDIA occupancy calculator" [19] applies. */
typedef struct {
    int cc_major, cc_minor, sm_count, warp_size;
    int regs_per_sm, regs_per_block, max_regs_per_thread, reg_alloc_unit, num_subpartitions;
    int max_threads_per_sm, max_threads_per_block, max_blocks_per_sm;
    int smem_per_sm, smem_per_block_optin, smem_reserved_per_block, smem_alloc_unit;
} orion_device_limits;

/* A kernel's resource usage at its natural ("original") build: Vreg and Vsmem of Eq. (1). */
typedef struct {
    int block_threads;      /* T, threads per CTA                                        */
    int regs_per_thread;    /* natural (uncapped) ptxas register count = MAXLIVE proxy   */
    int static_smem_bytes;  /* __shared__ arrays                                         */
    int dyn_smem_bytes;     /* the kernel's own dynamic shared-memory need (its tile)    */
    int min_reg_cap;        /* lowest register cap allowed (default 16)                  */
} orion_kernel_resources;

/* One occupancy level: k = ctas_per_sm resident CTAs per SM. */
typedef struct {
    int ctas_per_sm;         /* k                                                          */
    int warps_per_sm;        /* k * ceil(T/32)                                             */
    int occupancy_permille;  /* floor(1000 * warps / max warps per SM)                     */
    int reg_cap;             /* ptxas --maxrregcount for this level; 0 = uncapped (natural) */
    int smem_pad_bytes;      /* extra dynamic shared memory that caps residency at k */
    int limiter;             /* ORION_LIM_* bits                                            */
    int carveout_kb;         /* per-SM shared-memory configuration requested for the level
                                (8 .. 228 KB; the rest of the 256 KB array is L1); 0 = left to
                                the driver.  For padded levels it is the configuration the
                                residency probe measured k in; unpadded levels may run in a
                                larger one chosen by the driver, which does not change k     */
} orion_level;

/* How a level's CTA count is realised (the paper's small- vs large-cache axis, P:L757-P:L761,
 * Table 3): MAX_SMEM pins the carveout at 228 KB whenever padding is needed (smallest L1);
 * MIN_CARVEOUT picks the smallest shared-memory configuration that still holds k CTAs and
 * pads within it (largest L1 for spills and cached loads). */
enum { ORION_REALISE_MAX_SMEM = 0, ORION_REALISE_MIN_CARVEOUT = 1 };

/* ---- occupancy levels (question 1; host-only, pure) -------------------------------------- */

/* Nominal B200 (cc 10.0, 148 SMs) limits -- the Eq. (1) inputs (P:L121-P:L127: registers,
 * shared memory and thread slots per SM) for planning without a GPU; the B200 figures are
 * BASELINE.json's north star (64K regs, 228 KB, 64 warps, 148 SMs), the granularities those of
 * the calculator the paper uses ([19]). */
orion_status orion_b200_limits(orion_device_limits *out);

/* Limits of CUDA device `device` read from the driver (cuDeviceGetAttribute): the same Eq. (1)
 * inputs (P:L121-P:L127) as orion_b200_limits, measured instead of assumed.  ORION_E_CUDA
 * without a driver / device. */
orion_status orion_query_limits(int device, orion_device_limits *out);

/* Eq. (1) evaluated with the calculator's granularities (P:L125-P:L127): CTAs/SM of a
 * kernel with T threads, `regs` registers/thread, `smem_static` + `smem_dyn` bytes/CTA,
 * and the shared-memory carveout pinned at the device maximum.  *limiter gets ORION_LIM_*
 * bits (may be NULL). */
orion_status orion_ctas_per_sm(const orion_device_limits *dev, int block_threads, int regs,
                               int smem_static, int smem_dyn, int *ctas, int *limiter);

/* All feasible occupancy levels k = 1..k_max of a kernel ("generate code at all
 * occupancy levels"), ascending k.  Level k is realised by a register cap R_k (0 = natural
 * if the natural count already admits k; else the largest multiple of 8 below it that
 * admits k) and, where the registers admit more than k, dynamic shared-memory
 * padding.  Pure function of its inputs.  Capacity protocol: capacity too small
 * -> ORION_E_CAPACITY with *n_out = the number needed.  `out` may be NULL if capacity = 0. */
orion_status orion_levels(const orion_device_limits *dev, const orion_kernel_resources *res,
                          orion_level *out, int capacity, int *n_out);
/* orion_levels with an explicit realisation mode (ORION_REALISE_*; the small- vs large-cache
 * axis of P:L757-P:L761, Table 3); orion_levels = MAX_SMEM.  Same k_max and register caps in
 * both modes; padding and carveout differ. */
orion_status orion_levels_ex(const orion_device_limits *dev, const orion_kernel_resources *res, int mode,
                             orion_level *out, int capacity, int *n_out);
/* orion_ctas_per_sm (Eq. (1) with granularities, P:L125-P:L127) under a carveout preference of
 * `carveout_pct` percent of the maximum shared memory (< 0: the default, treated as the
 * maximum), rounded up to a configuration and raised to fit one CTA, as the driver does
 * (reading R-CARVE). */
orion_status orion_ctas_per_sm_carveout(const orion_device_limits *dev, int block_threads, int regs,
                                        int smem_static, int smem_dyn, int carveout_pct, int *ctas,
                                        int *limiter);

/* ---- code generation (question 1; host-only, no GPU needed) ------------------------------ */

/* The kernel's natural resources -- Vreg, Vsmem of Eq. (1) (P:L121-P:L127) and MAXLIVE's proxy
 * for Fig. 8 (reading R-A5) -- from compiling its PTX once, uncapped, with the embedded
 * ptxas (the "original" build).  Kernel ids (the paper's benchmarks, Table 2 P:L725-
 * P:L739; their math per readings R-O2, R-O3, R-SRAD):
 *   imageDenoising KNN: "knn_f4" (T = 128 / 256 / 64), "knn_f4_p1" (one pixel per
 *       thread, same bits), "knn_f4_t16" (the 49 taps of a pixel over 16 lanes: single small frames; C1 runs batches
 *       of frames through "knn_f4" at T = 256);
 *   imageDenoising NLM: "nlm_f4_w" (box sums + symmetric pairs, 3 pairs per pass,
 *       128-column tiles; the C2 / C5 default), "nlm_f4" (same, 122-column tiles),
 *       "nlm_f4_direct" (the direct 2401-term definition, cross-check form), "nlm_f4_regheavy"
 *       (direct form, centre patch in registers: the register-heavy C4 kernel; T = 128 / 64);
 *   hotspot: "hotspot_f32" (one step per launch; T = 256 / 128), "hotspot2h_f32" (two
 *       steps per launch, whole halo lanes), "hotspot4h_f32" (four steps per launch as a 4-stage
 *       register pipeline; the C3 default) -- width % 4 == 0 for the multi-step forms;
 *   srad: "srad_f32hs" (float4 strips, whole halo lanes, the ROI statistics fused in;
 *       width % 4 == 0; the default), "srad_f32h" (the same strips after a separate statistics
 *       kernel),
 *       "srad_f32" (register-sliding, any width), "srad_f32_tile" (shared-memory form; both
 *       cross-check forms, same bits).
 * block_threads = 0 selects the kernel's default CTA size.  ORION_E_INVALID for an unknown id /
 * CTA size, ORION_E_COMPILE when ptxas fails.  Host-only. */
orion_status orion_kernel_probe(const char *kernel_id, int block_threads, orion_kernel_resources *out);

/* Compile the kernel at register cap `reg_cap` (0 = uncapped) and report what ptxas did:
 * registers used, spill store / load bytes, local (stack) bytes per thread -- the spill cost a
 * register-capped level pays ("avoid excessive spilling"; C4's trade-off).  Memoised per
 * (kernel, T, cap).  Host-only; ORION_E_COMPILE with the ptxas log in orion_last_error(). */
orion_status orion_compile_info(const char *kernel_id, int block_threads, int reg_cap, int *regs,
                                int *spill_store_bytes, int *spill_load_bytes, int *local_bytes);

/* ---- multi-version binary (question 1; device) -------------------------------------------- */

typedef struct orion_variants orion_variants;   /* opaque, library-owned */

/* Build one sm_100a variant per level (the paper's "multi-version binary"):
 * the kernel's PTX is compiled once (at library build time) and assembled by ptxas once
 * per distinct register cap; every variant is loaded on `device`, its padding recomputed
 * from the ACTUAL register count, the carveout pinned when padding is used, and its
 * realised CTAs/SM checked twice: with cuOccupancyMaxActiveBlocksPerMultiprocessor and by a
 * residency probe launch of the function itself (every CTA counts the CTAs resident on its
 * SM; the driver may run a padded launch in a larger carveout configuration than requested,
 * which the API does not model).  A level whose planned configuration does not measure k is
 * retried in each larger configuration; none -> ORION_E_OCCUPANCY_MISMATCH.  The probe
 * launches (148 x 32 CTAs, ~1 ms) run on the legacy default stream during the build; they
 * also load every module (no lazy loading inside a later timed launch).  orion_sweep warms
 * and times each level once more before its timed rounds. */
orion_status orion_build_variants(int device, const char *kernel_id, int block_threads,
                                  const orion_level *levels, int n, orion_variants **out);
/* Number of variants (= levels) of the multi-version binary. */
orion_status orion_variants_count(const orion_variants *v, int *n);
/* The realised level (pad recomputed from actual registers) of variant `level_idx`. */
orion_status orion_variant_level(const orion_variants *v, int level_idx, orion_level *out);
/* What ptxas and the hardware did with variant `level_idx` (P:L215, P:L227-P:L229 realising a
 * level): registers, spill store / load bytes and local bytes per thread, and
 * verified_ctas_per_sm = the residency MEASURED by the probe launch (equal to the level's k).
 * Any output pointer may be NULL.  ORION_E_INVALID for a bad index. */
orion_status orion_variant_info(const orion_variants *v, int level_idx, int *regs, int *spill_store_bytes,
                                int *spill_load_bytes, int *local_bytes, int *verified_ctas_per_sm);
/* The kernel's natural resources (what orion_kernel_probe returned when building; Eq. (1)'s
 * Vreg / Vsmem, P:L121-P:L127). */
orion_status orion_variants_resources(const orion_variants *v, orion_kernel_resources *out);
void orion_variants_destroy(orion_variants *v);

/* ---- launching one iteration ------------------------------------------------------------ */

/* One launch of the kernel = one application iteration.
 *  denoisers: src = float4 rows [src_row_begin, src_row_end); dst = float4 rows
 *             [dst_row_begin, ...); output rows [row_begin, row_end) are computed.  src must
 *             hold every row the window + patch reach after clamping to [0, height) (halo:
 *             3 rows KNN, 6 rows NLM).  fparam[0] = Noise (1/h^2), fparam[1] = lerpC,
 *             fparam[2] = weight threshold, fparam[3] = lerp threshold (fraction of the 49
 *             window taps), as in the SDK imageDenoising sample (reading R-O2).
 *  hotspot:   src = T (float), aux = power (same rows as src), dst = T'; fparam[0..4] =
 *             sdc (step/Cap), rx = 1/Rx, ry = 1/Ry, rz = 1/Rz, amb (reading R-O3/R-A15).
 *             src must hold rows row_begin-S .. row_end+S-1 (clamped; S = steps per launch).
 *  halo exchange ("hotspot4h_f32", n_fanout = 2): a launch on a row band [row_begin, row_end)
 *             of a row-sharded grid also stores its first 4 and last 4 output rows -- the rows the
 *             neighbouring bands' next 4-step launch reads as halo -- into fanout[0] (upper
 *             neighbour) and fanout[1] (lower neighbour): device pointers such that global row y
 *             lands at fanout[f] + y * width (the neighbour's next input buffer, its own memory or
 *             a peer's over NVLink); NULL at the grid's top / bottom edge.  n_fanout other than 0
 *             or 2 -> ORION_E_INVALID.
 *  fan-out (every box-sum NLM kernel "nlm_f4*" except "nlm_f4_direct", every KNN kernel
 *             "knn_f4*"; not "nlm_f4_regheavy"): every output
 *             pixel is also stored into fanout[0 .. n_fanout) -- full width x height images
 *             (global row y at y * width), device pointers in this GPU's memory or a peer's
 *             reachable over NVLink (P2P / symmetric memory) -- so a row-sharded frame is
 *             gathered by the kernel's own epilogue as each tile completes (C5).  n_fanout = 0:
 *             no fan-out; > 8, or > 0 for other kernels -> ORION_E_INVALID.
 *  flags:     0, or ORION_ARGS_INDEPENDENT for a denoiser launch independent of the kernels
 *             enqueued before it on the stream since the last launch without the flag: it reads
 *             nothing they write and writes nothing they read (writes of identical values to the
 *             same words excepted) -- e.g. the next frame of a stream of frames, each in its own
 *             buffers (a pool reused round-robin rewrites a frame's output with the same bits);
 *             one band after another of orion_tune_split.  With programmatic dependent launch on
 *             (orion_set_pdl), the kernel then does not wait for its predecessor: its CTAs fill
 *             the previous grid's last wave (one frame per iteration, P:L605-P:L607, overlapped
 *             on the GPU), and a graph of such launches (orion_tuner_capture) keeps programmatic
 *             edges, so consecutive small frames run concurrently.  The caller asserts the
 *             independence; the result bits are the same.  Set on a
 *             stencil / SRAD launch (each reads its predecessor's output), or any other bit ->
 *             ORION_E_INVALID.  The host-buffer entry points (orion_tune_step_host,
 *             orion_host_pipe_submit) launch after their own copies and ignore it.
 *  chain:     NULL, or an orion_chain of this kernel family and grid (below): the launch is the
 *             chain's next iteration and waits for the previous one tile by tile, not grid-wide.
 *  batch:     0 or 1: one frame.  B > 1 (denoisers only, up to 65535): B whole frames of
 *             width x height pixels, stacked in src and in dst (frame f at f * width * height),
 *             filtered by one launch (grid z = frame) -- the small frames of configuration C1
 *             (BASELINE.json configs[0]) one batch per iteration of the tuner, whose
 *             work-normalised timing counts all B frames.  Requires row_begin =
 *             src_row_begin = dst_row_begin = 0 and row_end = src_row_end = height, no fan-out,
 *             no chain; otherwise ORION_E_INVALID.  The host-buffer entry points
 *             (orion_tune_step_host, orion_host_pipe_submit) copy the B frames as one block each
 *             way (a pipe needs max_rows >= B * height). */
#define ORION_ARGS_INDEPENDENT 1
typedef struct orion_chain orion_chain;   /* opaque, library-owned: see orion_chain_create */
typedef struct {
    const void *src;
    void *dst;
    const void *aux;
    int width, height;
    int row_begin, row_end;
    int src_row_begin, src_row_end;
    int dst_row_begin;
    float fparam[8];
    void *fanout[8];
    int n_fanout;
    int flags;
    orion_chain *chain;   /* NULL, or the chain this launch continues (orion_chain_create) */
    int batch;            /* 0 / 1: one frame; B > 1: B whole frames in one launch (below)     */
} orion_args;

/* ---- chains: consecutive stencil iterations overlapped tile by tile ----------------------
 * A stencil iteration reads what the previous one wrote, so each launch normally waits for the
 * whole previous grid (griddepcontrol.wait): the last, partial wave of every iteration leaves
 * SMs idle.  A chain (one kernel family, one whole grid, one stream) replaces that wait by
 * per-tile completion epochs in device memory: with programmatic dependent launch on, the CTA
 * at tile (x, y) of iteration n+1 starts as soon as the tiles of iteration n whose output it
 * reads or whose input it overwrites (the 3 x 3 neighbourhood: halos are smaller than a tile;
 * for "srad_f32hs" also the ROI tiles that write the statistics slots) have completed, so
 * iteration n+1 fills iteration n's last wave (the iterations of P:L605-P:L607, overlapped;
 * the bits are unchanged).  Chainable: "hotspot4h_f32", "srad_f32hs".  Rules: every launch of
 * the chain covers the whole grid (row_begin = 0, row_end = height, src / dst rows from 0),
 * takes no flags or fan-out, goes to the same stream, and is not captured into a graph
 * (orion_tuner_capture) or repeated by orion_sweep -- each gets ORION_E_INVALID.  Behind any
 * other liborion kernel on the stream (or at the chain's first launch) a chained launch waits
 * grid-wide as usual; kernels from outside liborion that use programmatic dependent launch
 * themselves must not be enqueued between two launches of a chain.  A CTA that waits 4 s
 * (a broken chain) traps instead of hanging. */
/* Allocates the chain's tile flags (zeroed) for `v`'s kernel family and a width x height grid
 * (the iterations of P:L605-P:L607 on one grid).  ORION_E_INVALID for a family without chains. */
orion_status orion_chain_create(const orion_variants *v, int width, int height, orion_chain **out);
/* Launches (iterations) enqueued on the chain so far, and its tile grid.  Any output may
 * be NULL. */
orion_status orion_chain_info(const orion_chain *c, unsigned *epoch, int *tiles_x, int *tiles_y);
/* Frees the chain (after its launches -- the iterations of P:L605 -- have completed). */
void orion_chain_destroy(orion_chain *c);

/* Launch variant `level_idx` (realising its occupancy level, P:L649, P:L757-P:L759) on
 * `stream` (async).  An empty row range (row_begin == row_end) is a no-op returning ORION_OK.
 * Every launch uses programmatic dependent launch unless it is disabled (ORION_PDL=0 in the
 * environment, or orion_set_pdl(0, ..)); results are the same bits either way. */
orion_status orion_launch(orion_variants *v, int level_idx, const orion_args *a, void *stream);

/* The method parameters of a kernel family, written into fparam[0 .. n) (n >= 8; the rest
 * zero) -- what orion_args.fparam holds for a launch with the defaults:
 *   "knn_f4*": Noise = 1/0.32^2, lerpC = 0.2, weight threshold 0.02, lerp threshold 0.79;
 *   "nlm_f4*": Noise = 1/1.45^2, 0.2, 0.10, 0.10  (CUDA-SDK imageDenoising [20], P:L91,
 *              the paper names the benchmark, not its math: reading R-O2);
 *   "hotspot*": sdc = step/Cap, rx, ry, rz, amb = 80 -- Rodinia hotspot ([6], Table 2
 *              P:L731) at the 512-grid's 31.25 um cell for every grid size (readings R-O3, R-A15);
 *   "srad*":   lambda = 0.5 (Rodinia srad_v2, Table 2; reading R-SRAD).
 * ORION_E_INVALID for an unknown id or n < 8.  Host-only. */
orion_status orion_default_params(const char *kernel_id, float *fparam, int n);

/* Launch plumbing of the P:L653 loop (not a method step): process-wide switch of
 * programmatic dependent launch for every later launch (initially
 * from ORION_PDL; default on).  `on` is 0 or 1 (else ORION_E_INVALID); *previous (may be
 * NULL) receives the setting it replaces.  A loop that will be replayed as a CUDA graph (graph
 * nodes are plain launches) turns it off so that the sweep times the levels the same way. */
orion_status orion_set_pdl(int on, int *previous);

/* Exhaustive occupancy sweep (Fig. 11's Orion-Min / Orion-Max methodology, P:L747-P:L755):
 * `rounds` rounds, each launching every level once in round-robin order (interleaving
 * cancels clock drift), each launch timed with a CUDA event pair on `stream`; writes the
 * median ms per level into ms_median[n levels].  A level whose (timed) warm-up launch is
 * shorter than 0.2 ms is timed over a batch of up to 64 back-to-back launches per sample and
 * reported per launch.  Synchronises the stream. */
orion_status orion_sweep(orion_variants *v, const orion_args *a, void *stream, int rounds, float *ms_median);

/* ---- runtime adaptation (question 2) ------------------------------------------------------ */

enum { ORION_DIR_DECREASING = -1, ORION_DIR_INCREASING = 1 };
enum { ORION_SELECT_FASTEST = 0, ORION_SELECT_LOWEST_WITHIN_TOL = 1 };

typedef struct {
    int maxlive_threshold;        /* Fig. 8 line 01: MAXLIVE >= 32 -> increasing (P:L645-P:L647)   */
    int samples_per_level;        /* timed launches per explored level (paper: 1)                  */
    int select_mode;              /* ORION_SELECT_* (reading R-A4)                        */
    int allow_direction_switch;   /* P:L689 fail-safe: switch direction if the original is final
                                     (default 1, reading R-A12)                           */
    float slowdown_tol;           /* Fig. 9 "Slowdown > .02?"                              */
    float worse_eps;              /* Fig. 9 "Worse runtime?" margin (paper: 0)                      */
    int expected_iterations;      /* canTune (Fig. 8 line 05): 0 = unknown (assume enough)          */
    int async_timing;             /* 0 (default, the paper's P:L653 loop): an exploring iteration
                                     synchronises on its event pair before returning.  1: it only
                                     records the pair; later iterations poll it (cuEventQuery) and,
                                     until it has completed, repeat the level being measured without
                                     timing it -- no host synchronisation anywhere, the measured
                                     launch runs back to back with its neighbours                   */
} orion_tuner_cfg;

/* The defaults: the paper's constants (MAXLIVE threshold 32; slowdown 0.02, P:L615;
 * worse_eps 0 and one sample per level) plus the readings' defaults (FASTEST, R-A4;
 * direction switch on, R-A12; synchronous timing). */
orion_status orion_tuner_default_cfg(orion_tuner_cfg *cfg);

typedef struct orion_tuner orion_tuner;   /* opaque, library-owned (holds CUDA events) */

/* Fig. 8 (P:L589-P:L603) applied to the variants' levels: direction from MAXLIVE (the
 * natural register count), ladder = original + conservative..max (increasing) or
 * original, original-1, .. 1 by padding (decreasing), with the opposite direction kept
 * as the fail-safe.  The tuner holds two CUDA events; ORION_E_INVALID for a bad cfg or
 * levels without the original (uncapped) version. */
orion_status orion_tuner_create(orion_variants *v, const orion_tuner_cfg *cfg, orion_tuner **out);

typedef struct {
    int iteration;        /* 0-based iteration index                                        */
    int level_idx;        /* variant launched this iteration                                 */
    int phase;            /* 0 = exploring (timed, synchronised), 1 = final (no host sync)   */
    int final_level_idx;  /* -1 until the final kernel is set                                */
    float ms;             /* measured kernel ms of this iteration while exploring, else -1;
                             async_timing: the measurement that completed during this call    */
} orion_step_report;

/* One application iteration under Fig. 9 (P:L605-P:L643, P:L651-P:L653, P:L687-P:L689):
 * first iteration runs the original; then the next ladder level while runtimes do not
 * degrade ("Worse runtime?" when increasing, "Slowdown > .02?" vs the best when
 * decreasing); then the final kernel every iteration.  Exploration iterations record a
 * CUDA event pair and synchronise on it; final iterations only enqueue the launch.  An empty
 * row range (row_begin == row_end) is not an iteration: nothing runs, *out reports
 * iteration = level_idx = phase = -1, ORION_OK. */
orion_status orion_tune_step(orion_tuner *t, const orion_args *a, void *stream, orion_step_report *out);
/* The measured time of an exploring iteration is work-normalised (ns per output element,
 * P:L975) before Fig. 9 compares it, so iterations of different sizes compare fairly. */

/* n consecutive Fig. 9 iterations (P:L605-P:L643), exactly n calls of orion_tune_step on
 * args[0..n-1] (host array of n
 * orion_args, caller-owned), issued from the library in one call: launch-bound frames (C1) do not
 * pay a foreign-function call per iteration.  *last (may be NULL) = the report of the last
 * iteration.  Errors: ORION_E_INVALID for NULL / n < 0; otherwise the first failing
 * orion_tune_step's status (the iterations before it have been issued). */
orion_status orion_tune_steps(orion_tuner *t, const orion_args *args, int n, void *stream, orion_step_report *last);

/* Kernel splitting ("we split one kernel invocation into multiple invocations, such
 * that every invocation of the split kernel launches a subset of the threads", [30]): the
 * output rows [row_begin, row_end) of ONE frame are processed as `bands` consecutive row
 * bands, each one orion_tune_step iteration, so a one-shot frame still gets tuned.  The
 * union of the bands equals one unsplit launch bit for bit.  reports[bands] may be NULL;
 * a band left empty by the rounding reports iteration = -1. */
orion_status orion_tune_split(orion_tuner *t, const orion_args *a, int bands, void *stream,
                              orion_step_report *reports);

/* Same iteration (Fig. 9, P:L605-P:L643) end to end from HOST buffers: copies a->src (host, pinned for async)
 * into dev_src, runs orion_tune_step with device pointers, copies dev_dst back into
 * a->dst (host) -- all on `stream`, then synchronises it.  dev_src / dev_dst are
 * caller-owned device buffers at least as large as the host regions (and dev_aux for the
 * stencil power map).  Byte counts copied are returned in *h2d_bytes / *d2h_bytes. */
orion_status orion_tune_step_host(orion_tuner *t, const orion_args *a, void *dev_src, void *dev_dst,
                                  void *dev_aux, void *stream, orion_step_report *out,
                                  long long *h2d_bytes, long long *d2h_bytes);

/* A whole iterative stencil run end to end from HOST buffers -- the Rodinia driver shape
 * (copy the grid in, iterate, copy it out), the iterations being the ones
 * Fig. 9 tunes across (P:L651-P:L653).  Kernels of kind hotspot ("hotspot_f32",
 * "hotspot2h_f32", "hotspot4h_f32") and srad ("srad_f32", "srad_f32h", "srad_f32hs", "srad_f32_tile") only, whole grids only
 * (a->row_begin = a->src_row_begin = a->dst_row_begin = 0, a->row_end = a->src_row_end =
 * a->height).
 *   a->src  host initial grid (fp32, width x height, row-major; pinned for async copies)
 *   a->aux  hotspot: host power map (same shape); srad: ignored
 *   a->dst  host buffer receiving the grid after `iterations` launches
 *   dev_a, dev_b  caller-owned device grids (ping-pong), width x height fp32 each
 *   dev_aux hotspot: device power map buffer (filled here); srad: the device float q0sqr
 *           ("srad_f32hs": unused, may be NULL -- dev_a / dev_b then hold width x height +
 *           ORION_SRAD_STATS_FLOATS floats each, and the slots of the initial grid are written
 *           once with orion_srad_stats_init before the first iteration)
 *   roi     srad only: {r1, r2, c1, c2} of the ROI statistics run before every iteration
 * Copies in, runs `iterations` orion_tune_step iterations on `stream` (hotspot2h_f32 advances
 * two time steps per iteration, hotspot4h_f32 four; chainable families run them as one
 * internal orion_chain), copies the final grid out and synchronises the stream.
 * Bytes copied are returned in *h2d_bytes / *d2h_bytes.  ORION_E_INVALID on other kernels,
 * partial row ranges or missing buffers. */
orion_status orion_tune_run_host(orion_tuner *t, const orion_args *a, int iterations, void *dev_a, void *dev_b,
                                 void *dev_aux, const int *roi, void *stream, long long *h2d_bytes,
                                 long long *d2h_bytes);

/* Pipelined end-to-end iterations from HOST buffers (the P:L653 tuned loop fed from the host:
 * what an application streaming frames sees; bench.py's e2e figure).  The pipe owns `depth` slots of device
 * staging buffers (width x max_rows elements each for src, dst and -- stencil -- aux;
 * allocated here, never in submit) and three non-blocking streams: the H2D copy of frame n,
 * the kernel of frame n-1 (orion_tune_step on the pipe's compute stream) and the D2H copy of
 * frame n-2 run concurrently (PCIe is full duplex).  Host buffers must be pinned and must
 * stay untouched until orion_host_pipe_drain returns.  Errors: ORION_E_INVALID when a frame
 * does not fit the pipe's width / max_rows; driver errors as ORION_E_CUDA. */
typedef struct orion_host_pipe orion_host_pipe;   /* opaque, library-owned */
/* Create a pipe over tuner t (its Fig. 9 walk, P:L605-P:L643, runs inside submit); depth 1..8. */
orion_status orion_host_pipe_create(orion_tuner *t, int width, int max_rows, int depth, orion_host_pipe **out);
/* Enqueue one tuned iteration (orion_tune_step, Fig. 9 P:L605-P:L643): a->src / a->aux /
 * a->dst are HOST pointers laid out as for
 * orion_launch (src rows [src_row_begin, src_row_end), dst rows from dst_row_begin).
 * Returns without waiting; bytes copied are reported in *h2d_bytes / *d2h_bytes. */
orion_status orion_host_pipe_submit(orion_host_pipe *p, const orion_args *a, orion_step_report *out,
                                    long long *h2d_bytes, long long *d2h_bytes);
/* Wait until every submitted iteration's output is in host memory (end of the P:L653 loop). */
orion_status orion_host_pipe_drain(orion_host_pipe *p);
/* Synchronise the pipe's streams and free its staging buffers, events and streams (SURVEY §8(b)
 * ownership: library-owned objects have a create / destroy pair). */
void orion_host_pipe_destroy(orion_host_pipe *p);

/* Current Fig. 8 candidate ladder (P:L589-P:L603): *direction (ORION_DIR_*), ladder level
 * indices (ladder[0] = the original) -> out[capacity]; capacity protocol as
 * orion_levels.  After a P:L689 direction switch it is the opposite ladder. */
orion_status orion_tuner_ladder(const orion_tuner *t, int *direction, int *out, int capacity, int *n_out);
/* The final kernel of Fig. 9 ("set final kernel"): its level index (-1 while exploring)
 * and the iteration it was set at. */
orion_status orion_tuner_final(const orion_tuner *t, int *final_level_idx, int *iterations_to_final);
/* The runtime table Fig. 9 has seen so far (P:L605-P:L643; work-normalised per P:L975):
 * out[i] = the value observed for level i -- ns per output element, the fastest of its
 * samples_per_level samples -- or -1 for a level not (yet) measured.  `n` must equal the
 * number of variants (ORION_E_INVALID otherwise).  Host-only read of tuner state; used to
 * replay a live walk through an independent Fig. 9 (the oracle's O4) and check that the
 * decisions are identical. */
orion_status orion_tuner_tried(const orion_tuner *t, float *out, int n);
/* Checkpoint / resume of the tuner's decision: a final level recorded from an
 * earlier run (orion_tuner_final, keyed by the caller on kernel id, device and shape) is set
 * directly, so a restarted application skips the Fig. 9 exploration.  ORION_E_INVALID for an
 * index outside the variants; ORION_E_STATE while an async measurement is in flight. */
orion_status orion_tuner_resume(orion_tuner *t, int final_level_idx);
void orion_tuner_destroy(orion_tuner *t);

/* ---- CUDA graph replay of settled iterations (launch-bound loops) ------------------------- */

typedef struct orion_graph orion_graph;   /* opaque, library-owned (a CUgraphExec) */

/* Once Fig. 9 has set the final kernel ("run final kernel" every later iteration), the
 * iterations are plain launches of one variant: capture `n` of them -- args[i] for iteration i,
 * e.g. a ring of frames; device pointers, geometry as for orion_launch -- into a CUDA graph on
 * a library stream.  Each orion_graph_launch then replays the n launches on `stream` with one
 * host call (no per-launch host work: what bounds small frames such as C1's 64x64).  The
 * tuner's iteration counter advances by n per replay.  The nodes are plain launches unless every
 * args[i] carries ORION_ARGS_INDEPENDENT and PDL is on: then they keep programmatic dependent
 * launch and overlap.  ORION_E_STATE while the tuner is still exploring; ORION_E_INVALID on
 * n < 1, bad args or chained args. */
orion_status orion_tuner_capture(orion_tuner *t, const orion_args *args, int n, orion_graph **out);
orion_status orion_graph_launch(orion_graph *g, void *stream);
void orion_graph_destroy(orion_graph *g);

/* Host-only replay of Fig. 8 + Fig. 9 on a synthetic per-level runtime table (no GPU):
 * levels[n] as from orion_levels, natural_regs = MAXLIVE proxy, ms_of_level[n] = the runtime
 * each level would take; runs `iterations` iterations writing the level index run at each
 * into ran[iterations], and the final level / the iteration it was set at. */
orion_status orion_tuner_replay(const orion_tuner_cfg *cfg, const orion_level *levels, int n, int natural_regs,
                                const float *ms_of_level, int iterations, int *ran, int *final_level_idx,
                                int *final_iteration);

/* ---- synthetic inputs on the device (the generator's GPU twin; no method arithmetic) ---- */

/* Rows [row_begin, row_end) of the W x H seeded noisy RGBA image into dst (pitch W): the device
 * twin of synth.noisy_rgba (SURVEY §8(d) generator; DESIGN §5 input recipe -- the paper
 * publishes no inputs, P:L85-P:L91), bit-identical to it, so a row slab of a sharded frame (C5)
 * is the same bits as those rows of the full image.  seed < 2^24. */
orion_status orion_generate_rgba(int device, void *dst, int width, int height, int row_begin, int row_end,
                                 unsigned seed, float sigma, void *stream);
/* Thermal T0 and power map (W x H) into t0 / power: the device twin of synth.thermal_inputs
 * (T0 = 323.15 + U[0,1) * 20, P = U[0,1) * 0.05; Rodinia hotspot's
 * inputs are unpublished).  Also SRAD's positive image. */
orion_status orion_generate_thermal(int device, void *t0, void *power, int width, int height, unsigned seed,
                                    void *stream);
/* SRAD's per-iteration ROI statistics (Rodinia srad_v2, reading R-SRAD; Table 2
 * P:L739): q0sqr = var / mean^2 of J over rows [r1, r2] x cols [c1, c2] (inclusive) of the
 * width-pitched device image J, reduced in double in a fixed order by one CTA and stored as
 * one float at device address q0 -- the `aux` of the "srad_f32" kernel's orion_args
 * (whose fparam[0] = lambda).  Asynchronous on `stream`. */
orion_status orion_srad_roi_stats(int device, const void *J, int width, int height, int r1, int r2, int c1, int c2,
                                  void *q0, void *stream);
/* SRAD with the ROI statistics fused into the update ("srad_f32hs"): every grid it reads or writes
 * is width x height floats FOLLOWED by ORION_SRAD_STATS_FLOATS floats of statistics slots (the
 * ROI's partial sums, in double).  A launch derives q0sqr (reading R-SRAD, Table 2) from
 * the slots behind src and writes its output ROI's slots behind dst, so an iteration is ONE
 * kernel (the tuner's iteration, P:L651-P:L653) instead of statistics + update.  Its orion_args:
 * whole grids (row ranges 0 .. height), fparam[0] = lambda, fparam[1..4] = r1, r2, c1, c2
 * (inclusive ROI, exact integers), aux unused; width % 4 == 0. */
#define ORION_SRAD_STAT_SLOTS 64
#define ORION_SRAD_STATS_FLOATS (4 * ORION_SRAD_STAT_SLOTS)
/* The first iteration's input: write the statistics slots of grid J (device, width x height +
 * ORION_SRAD_STATS_FLOATS floats) for ROI rows [r1, r2] x cols [c1, c2] in "srad_f32hs"'s
 * partition, asynchronously on `stream` (reading R-SRAD's ROI statistics).
 * ORION_E_INVALID for a ROI outside the grid or spanning more than ORION_SRAD_STAT_SLOTS
 * (42-row strip, 120-column block) slots, or width % 4 != 0. */
orion_status orion_srad_stats_init(int device, void *J, int width, int height, int r1, int r2, int c1, int c2,
                                   void *stream);
/* Write `bytes` of `buf` (a device scratch buffer larger than L2) to evict the L2: a
 * measurement utility (cold-cache timing, SURVEY §8(d) timing protocol); no method math. */
orion_status orion_flush_l2(int device, void *buf, long long bytes, void *stream);

/* ---- diagnostics (SURVEY §5 failure detection; not method steps) ---------------------------- */
/* Name of a status code ("ORION_OK", "ORION_E_INVALID", ...). */
const char *orion_status_str(orion_status s);
/* The calling thread's last error message (driver string, ptxas log, argument check). */
const char *orion_last_error(void);
/* Number of kernel launches liborion has enqueued in this process (all kernels; graph replays
 * count their captured launches): the evidence bench.py reports as gpu_launches. */
long long orion_launch_count(void);
/* Library name and version string. */
const char *orion_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ORION_H */
