/* fpmpmm.h -- C ABI of libfpmpmm.so: FPM-partitioned column-based parallel
 * matrix multiplication on B200 (sm_100a).
 *
 * Method: Zhong, Rychkov, Lastovetsky, "Data Partitioning on Heterogeneous
 * Multicore and Multi-GPU Systems Using Functional Performance Models of
 * Data-Parallel Applications", Cluster 2012.  Citations "P:<line>" refer to
 * the paper text; "Q<n>" to the readings listed in DESIGN.md.
 *
 * The application "takes the FPMs of heterogeneous processors as input,
 * partitions the matrices using the FPM-based data partitioning algorithm, and
 * performs the blocked matrix multiplication, using the GEMM kernel".
 * The four calls of that statement are fpm_sample, fpm_partition,
 * colpart_arrange and pmm_run.
 *
 * Conventions
 *  - Every function returns an int status: FPM_OK (0) on success, a negative
 *    FPM_E* code on failure.  No C++ exception crosses the ABI.  The message of
 *    the last failure on the calling thread is returned by fpm_last_error().
 *  - "blocks" are b x b blocks of the N x N matrices; n = N / b, T = n * n.
 *  - Host matrices are row-major.  Pointers passed in are owned by the caller,
 *    read (or written) only for the duration of the call; the library never
 *    keeps them.
 *  - The library owns everything it allocates inside a pmm_ctx (device
 *    buffers, streams, events, IPC mappings, NCCL communicators); all of it is
 *    released by pmm_destroy.
 *  - fpm_partition, colpart_arrange, colpart_arrange_fpm, colpart_plan_step
 *    and fpm_model_speed are pure host functions: no GPU, no context,
 *    thread-safe.  Calls on one
 *    pmm_ctx must be serialised by the caller.
 */
#ifndef FPMPMM_H
#define FPMPMM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FPM_OK            0
#define FPM_EINVAL       -1   /* invalid argument (shape, model, arrangement, ...) */
#define FPM_ENOMEM       -2   /* host or device allocation failed                 */
#define FPM_ECUDA        -3   /* CUDA runtime / driver error (message has detail)  */
#define FPM_ENCCL        -4   /* NCCL error                                        */
#define FPM_EUNSUPPORTED -5   /* configuration not supported (e.g. SM cap)         */
#define FPM_ESTATE       -6   /* call out of order (e.g. pmm_compute before setup) */

#define FPM_MAX_DEVICES  16

typedef enum { FPM_F32 = 0, FPM_F64 = 1 } fpm_dtype;
typedef enum { FPM_DIST_PM1 = 0, FPM_DIST_INT = 1 } fpm_dist;

/* Functional performance model of one device (P:8 "represents the processor
 * speed by a function of problem size"; P:18 built from timed kernel runs on
 * sqrt(x) x sqrt(x) submatrices).  x[j]: problem size in blocks, strictly
 * increasing, >= 1.  s[j]: speed in flop/s, finite, > 0.  npts >= 1.
 * Evaluation (reading Q4): piecewise linear in s between points, constant
 * beyond both ends; t(x) = x / s(x). */
typedef struct {
    int32_t        npts;
    const int64_t* x;
    const double*  s;
} fpm_model;

/* One device's rectangle of the column-based arrangement (Fig. 1(a)),
 * in blocks: column index `col` (-1 for an empty rectangle), top-left block
 * (row0, col0), height h and width w. */
typedef struct {
    int32_t col;
    int64_t row0, col0, h, w;
} colpart_rect;

/* One pivot transfer of iteration k (reading Q12), in blocks.
 * A moves: device src sends rows [begin, end) of block-column k to dst.
 * B moves: device src sends cols [begin, end) of block-row k to dst.
 * src == dst marks a local use (no transfer). */
typedef struct {
    int32_t src, dst;
    int64_t begin, end;
} colpart_move;

/* Statistics of one pmm_compute / pmm_run.  Times in seconds, measured with
 * CUDA events on the launching streams. */
typedef struct {
    double  t_compute_s;                        /* k-loop, first event to last, max over devices  */
    double  t_upload_s;                         /* host -> device scatter (pmm_run only)          */
    double  t_download_s;                       /* device -> host gather  (pmm_run only)          */
    double  per_dev_compute_s[FPM_MAX_DEVICES]; /* sum of split + update kernel time per device   */
    double  per_dev_update_s[FPM_MAX_DEVICES];  /* sum of rank-b update kernel time per device    */
    double  gflops;                             /* 2 N^3 / t_compute_s / 1e9                      */
    double  imbalance;                          /* max/mean - 1 of per_dev_compute_s (area > 0)   */
    int64_t iters;                              /* n = N / b                                      */
    int64_t comm_bytes;                         /* pivot bytes received by this process's devices */
    int64_t kernel_launches;                    /* library kernels launched in the k-loop         */
    int64_t updates;                            /* rank-(f b) update launches (f pivots fused)    */
    int64_t ooc_devices;                        /* bit i: device i held C_i out of core           */
    int64_t ooc_bytes;                          /* C bytes streamed host <-> device (out of core) */
    double  per_dev_span_s[FPM_MAX_DEVICES];    /* k-loop start to the device's last update end:
                                                   when it finished (staging that overlaps its
                                                   updates counted once)                        */
} pmm_stats;

typedef struct pmm_ctx pmm_ctx;

/* ---------------------------------------------------------------- misc */
const char* fpm_last_error(void);  /* thread-local, never NULL */
int32_t     fpm_abi_version(void); /* 1 */

/* ------------------------------------------------ host algorithms (pure) */

/* s(x) of one model (P:8, reading Q4).  FPM_EINVAL if the model is invalid
 * or x < 0. */
int fpm_model_speed(const fpm_model* model, int64_t x, double* s_out);

/* FPM-based data partitioning (P:9 "all processors complete their work
 * within the same time"; algorithm of [5]; readings Q1-Q3).
 * Computes integer areas d[0..p) with sum d = total_blocks such that the
 * times d_i / s_i(d_i) are balanced, by the geometric method: bisection of
 * the line through the origin (slope = 1 / time) over the speed graphs,
 * followed by an exact integer phase.  The result is bit-identical to the
 * canonical definition (give blocks one at a time to the device with the
 * smallest t_i(d_i + 1), ties to the lowest index), which is min-max optimal
 * whenever each t_i is non-decreasing.
 * models: p entries (1 <= p <= FPM_MAX_DEVICES).  d_out: p int64, written.
 * iters_out (nullable): bisection iterations used.
 * Errors: FPM_EINVAL on p out of range, total_blocks < 0, invalid model. */
int fpm_partition(int64_t total_blocks, int32_t p, const fpm_model* models,
                  int64_t* d_out, int32_t* iters_out);

/* Column-based arrangement ("arranges the submatrices to be as square as
 * possible, minimising the total volume of communications"; [17] P:144;
 * reading Q10): rectangles of areas close to d_i tiling the n x n grid,
 * minimising the sum of half-perimeters.  d: p areas with sum = n*n.
 * rects_out: p entries.  Achieved areas h_i * w_i differ from d_i by the
 * integer rounding of widths/heights.  Zero areas give empty rectangles
 * (col = -1).  Errors: FPM_EINVAL if sum d != n*n, any d < 0, n < 1. */
int colpart_arrange(int64_t n, int32_t p, const int64_t* d, colpart_rect* rects_out);

/* Column-based arrangement whose integers come from the FPMs (reading Q25 in
 * DESIGN.md).  P:9 "all processors complete their work
 * within the same time" applied to the integer rectangles themselves instead
 * of rounding continuous quotas: for every split of the devices, sorted by
 * (-d_i, i), into consecutive columns, each column's heights (sum n) and then
 * the columns' widths (sum n) are given out one unit at a time to whichever
 * device / column would finish it earliest under the models; the split with
 * the smallest (predicted makespan, sum of half-perimeters, #columns, column
 * sizes) is returned.  Removes the rounding imbalance of colpart_arrange
 * (e.g. 132 vs 128 blocks at n = 32, p = 8 equal devices).
 * d: p areas with sum = n*n (they fix the device order and which devices take
 * part); models: p speed functions as for fpm_partition.  rects_out: p
 * entries; devices left without area get (-1, 0, 0, 0, 0); columns of positive
 * width are numbered 0.. left to right.  Cost O(q^3 n^2) model evaluations for
 * q devices with d_i > 0.  Errors: FPM_EINVAL if sum d != n*n, any d < 0,
 * n outside [1, 1024], p out of range, invalid model. */
int colpart_arrange_fpm(int64_t n, int32_t p, const int64_t* d, const fpm_model* models,
                        colpart_rect* rects_out);

/* Delivery plan of iteration k ("pivot column of matrix A and pivot row
 * of matrix B are broadcast horizontally and vertically"; reading Q12).
 * Writes at most a_cap / b_cap moves, sorted by (src, dst, begin); the counts
 * are always written.  FPM_EINVAL if the rectangles do not tile the grid, k
 * out of range, or a capacity is too small (counts still written). */
int colpart_plan_step(int64_t n, int32_t p, const colpart_rect* rects, int64_t k,
                      colpart_move* a_moves, int32_t a_cap, int32_t* a_count,
                      colpart_move* b_moves, int32_t b_cap, int32_t* b_count);

/* ------------------------------------------------------------- runtime */

/* Single-process context driving p "devices".  Device i runs on CUDA ordinal
 * cuda_devices[i]; several devices may share one GPU.  sm_caps (nullable):
 * 0 = the whole GPU, else a cap on SMs (even, >= 2) for heterogeneity
 * emulation (BASELINE north_star): the persistent rank-b update kernel, which
 * holds one SM per CTA, runs with a grid of `cap` CTAs.  Pivot
 * transfers between devices are device-to-device copies on the receivers'
 * communication streams.
 *
 * cuda_devices[i] = FPM_CPU_DEVICE makes device i a host-CPU device (PAPER.md
 * a socket of c cores executing the GEMM kernel
 * simultaneously): sm_caps[i] = c cores (0 = every core left), taken as
 * consecutive cores of the process's affinity mask after those of earlier CPU
 * devices -- and after the first core when the context drives GPUs (a
 * core dedicated to the GPU); pmm_set_device_option "cpu_first_core" moves
 * them.  Its A_i, B_i, C_i live in host memory (pinned and mapped when GPUs
 * are present: their staging kernels read its pivots directly); its update is
 * the host GEMM of fpm_k_cpu_gemm on its c pinned cores, rows split evenly;
 * its k-loop runs on a thread of its own, concurrently with the GPU devices'
 * streams, pulling pivots held by GPU devices device -> host one update group
 * ahead.  A CPU device is a device of the partition chosen by the caller,
 * never a fallback: GPU devices' updates always run on their GPUs.  Contexts
 * with only CPU devices need no GPU.  Not available in NCCL / IPC contexts.
 * fpm_sample(dev = -1) on a context with CPU devices runs every device on a
 * host thread of its own, all repetitions in step: each device runs its kernel
 * for the same wall-clock window (>= 4 runs of the slowest) and its speed is
 * its completed runs over that time (P:10 (ii) synchronised measurement).
 * Errors: FPM_EINVAL, FPM_ECUDA, FPM_EUNSUPPORTED (SM cap or cores not
 * available). */
#define FPM_CPU_DEVICE (-1)
int pmm_create_local(int32_t p, const int32_t* cuda_devices, const int32_t* sm_caps,
                     pmm_ctx** out);

/* Multi-process context: one process per GPU (rank `rank` of `world`), pivot
 * broadcasts over NCCL (libnccl.so.2 loaded at run time): vertical B pivot
 * rows with ncclBroadcast on per-column communicators, horizontal A pivot
 * slices with grouped ncclSend/ncclRecv.  nccl_id: 128 bytes from
 * pmm_nccl_unique_id() on rank 0, distributed by the caller. */
int pmm_nccl_unique_id(uint8_t id_out[128]);
int pmm_create_nccl(int32_t rank, int32_t world, int32_t cuda_device, int32_t sm_cap,
                    const uint8_t nccl_id[128], pmm_ctx** out);

/* Multi-process context without NCCL: one process per GPU (rank of world),
 * pivots pulled one-sidedly from the peers' resident A_q / B_q through CUDA IPC
 * mappings (NVLink for peers on other GPUs), fused into the staging kernels that
 * split them for the tensor cores.  The inputs never change during the
 * iteration loop, so pulls need no synchronisation with the owner.  Protocol:
 * pmm_setup -> pmm_ipc_export (every rank) -> all-gather of the blobs by the
 * caller -> pmm_ipc_import -> pmm_upload / pmm_fill_synthetic -> caller
 * barrier -> pmm_compute -> pmm_download; or, after the import, pmm_run on
 * every rank with its own host window (same problem, else FPM_EUNSUPPORTED):
 * each rank streams its panels in and writes a 64-bit upload-progress flag per
 * pivot, and a peer pulls a pivot only after that flag shows it landed.
 * Failure detection: a k-loop that cannot finish because a peer stopped (its
 * flag never advances) fails with FPM_ECUDA instead of blocking -- the host
 * wait gives up after FPM_IPC_TIMEOUT_S seconds (env, default 600, 0 = never)
 * and the update kernel's staging warps trap after 60 s of waiting. */
#define FPM_IPC_BLOB_BYTES 256
int pmm_create_ipc(int32_t rank, int32_t world, int32_t cuda_device, int32_t sm_cap, pmm_ctx** out);
int pmm_ipc_export(pmm_ctx* ctx, uint8_t blob_out[FPM_IPC_BLOB_BYTES]);
/* blobs: world x FPM_IPC_BLOB_BYTES, rank order. */
int pmm_ipc_import(pmm_ctx* ctx, const uint8_t* blobs, int32_t world);

int pmm_destroy(pmm_ctx* ctx);

/* Fix the problem: N x N matrices, blocking factor b ("blocking factor
 * b"), arrangement rects[p] (p = devices of the context, or world size in
 * NCCL mode), dtype.  Allocates the resident A_i, B_i, C_i of the devices this
 * process drives plus pivot staging.  Requires b | N, b % 32 == 0 (FP32) or
 * b % 8 == 0 (FP64), rects tiling the n x n grid.
 * Layout in HBM: A_i as w_i block-columns, each (h_i b) x b row-major
 * (K-major pivot panels); B_i as h_i block-rows, each b x (w_i b) row-major;
 * C_i (h_i b) x (w_i b) row-major. */
int pmm_setup(pmm_ctx* ctx, int64_t N, int64_t b, int32_t p, const colpart_rect* rects,
              fpm_dtype dt);

/* Copy this process's rectangles of A and B from host windows (untimed
 * distribution, P:8 "Data partitioning algorithms map all data to processors
 * and do not redistribute it").  The host arrays hold the global rows
 * [row_base, ...) and columns [col_base, ...) with leading dimension ld
 * (elements); every local rectangle must lie inside the window.  Element type
 * = the dtype of pmm_setup.  Zeroes C_i. */
int pmm_upload(pmm_ctx* ctx, const void* A, const void* B, int64_t ld,
               int64_t row_base, int64_t col_base);

/* Fill the resident A_i, B_i with the seeded counter-based generator of
 * synth/__init__.py (global element index row*N + col), zero C_i. */
int pmm_fill_synthetic(pmm_ctx* ctx, uint64_t seed_a, uint64_t seed_b, int32_t dist);

/* Run the N/b iterations on resident data: per iteration pivot exchange
 * (look-ahead one iteration, on communication streams) and the rank-b update
 * C_i += A(b) x B(b) on each device.  Iteration 0 writes C_i = A(0) B(0)
 * (no zeroing pass), so every call leaves C_i = (A B)_i.  zero_c is accepted
 * for compatibility and has no effect.  Blocks until done. */
int pmm_compute(pmm_ctx* ctx, int32_t zero_c, pmm_stats* stats);

/* pmm_compute, then C_i into a host window (convention of pmm_download), with
 * the device -> host copy overlapped with the last updates: the last L update
 * groups (option "e2e_tail") run band-major over rows of C_i, and each band is
 * copied out as soon as it is final.  Every element still receives the
 * updates in k order.  Devices without a tail (FP64, out-of-core) are copied
 * after the loop.  stats->t_download_s = copy time after the last update. */
int pmm_compute_into(pmm_ctx* ctx, void* C, int64_t ld, int64_t row_base, int64_t col_base,
                     pmm_stats* stats);

/* Copy this process's C_i into a host window (same convention as upload). */
int pmm_download(pmm_ctx* ctx, void* C, int64_t ld, int64_t row_base, int64_t col_base);

/* Copy the global block C[r0 : r0+rows, c0 : c0+cols] (must lie inside one
 * rectangle held by this process) into host memory (row stride ld elements).
 * For sampled checks at full size without gathering all of C. */
int pmm_download_block(pmm_ctx* ctx, int64_t r0, int64_t c0, int64_t rows, int64_t cols, void* C_host,
                       int64_t ld);

/* Timeline of the last k-loop on local GPU device `dev` (arrangement index),
 * per update group g (f pivots fused, in k order): out[4g .. 4g+3] = start and
 * end of its staging (pivot exchange + pack) and start and end of
 * its rank-(f b) update (a7), in seconds after the loop's start event, from the
 * CUDA events on the device's streams -- the per-iteration view behind the
 * Fig. 6 computation times.  Groups of a download-overlapped tail or
 * of a phase the loop did not time are NaN.  out: cap doubles (caller-owned;
 * 4 per group); *count = number of groups (written even when cap is short).
 * Blocks until the loop finished.  FPM_EINVAL for a CPU device or one this
 * process does not drive; FPM_ESTATE before pmm_setup. */
int pmm_group_times(pmm_ctx* ctx, int32_t dev, double* out, int32_t cap, int32_t* count);

/* Whole call on host matrices: setup (if the problem changed), then the N/b
 * iterations with the inputs streamed from the host windows (block-column k of
 * A and block-row k of B are copied host -> device on the communication stream
 * just ahead of iteration k, overlapping earlier updates), then the download
 * of C, overlapped with the last updates as in pmm_compute_into.  A, B, C are host windows as for pmm_upload (pinned memory gives
 * asynchronous copies).  stats: t_compute_s includes the streamed upload,
 * t_upload_s = time until the last panel landed, t_download_s. */
int pmm_run(pmm_ctx* ctx, const void* A, const void* B, void* C, int64_t N, int64_t b,
            int32_t p, const colpart_rect* rects, fpm_dtype dt, int64_t ld,
            int64_t row_base, int64_t col_base, pmm_stats* stats);

/* Build a speed function (P:9 kernel-based benchmarking, P:10 (iii) repeated
 * until statistically reliable, P:18 sqrt(x) x sqrt(x) submatrices): for each
 * x = sizes[j] (must be a perfect square m^2), time the computational kernel
 * C += A(b) x B(b) (pivot split + rank-b update, as the k-loop runs it: where
 * its updates stage the next group in-kernel -- option "fused_staging" -- the
 * timed update stages the next run's operands the same way) on an (m b) x (m b)
 * C on device `dev` of the context (its SM cap applies) and return
 * speeds_out[j] = 2 x b^3 / t in flop/s.  Repeats until the 95% confidence
 * half-width is <= 2.5% of the mean (>= 5, <= 50 repetitions, reading Q8).
 * dev = -1 samples every device of the context simultaneously (P:10 (ii)
 * "processes are synchronised", so shared resources are contended as in the
 * run): after the warm-ups each device runs its kernel k_i = round(t_max /
 * t_i) times (<= 64) per repetition, so all stay busy for the same window, and
 * a run's time is the window / k_i.  The outputs are then p x nsizes,
 * device-major.
 * rel_ci95_out / reps_out nullable. */
int fpm_sample(pmm_ctx* ctx, int32_t dev, fpm_dtype dt, int64_t b, const int64_t* sizes,
               int32_t nsizes, double* speeds_out, double* rel_ci95_out, int32_t* reps_out);

/* The same timing procedure on rectangles: shapes = nshapes (h, w) pairs in
 * blocks (C of h b x w b; speeds_out[j] = 2 h w b^3 f / t, attributed to the
 * area x = h w).  P:18: the speed "does not vary with the nearly square shapes
 * of submatrices", so the rectangles a column arrangement hands out are valid
 * sample points of the FPM -- the operating-point refinement of reading Q26
 * samples each device at its own rectangle.  dev = -1: every device of the
 * context at once, each on its own shapes (shapes device-major, p x nshapes x 2;
 * outputs p x nshapes), i.e. under the contention of the run.  CPU devices
 * (dev >= 0 only) and out-of-core GPU sizes are sampled as by fpm_sample. */
int fpm_sample_rects(pmm_ctx* ctx, int32_t dev, fpm_dtype dt, int64_t b, const int64_t* shapes,
                     int32_t nshapes, double* speeds_out, double* rel_ci95_out, int32_t* reps_out);

/* Tuning / selection knobs (all optional):
 *   "f32_scheme": -1 = auto (default) = 0.  0 = F16X3 (x 2^e = h0 + h1, both
 *                 fp16, 2^e a per-row / per-column power of two; 3 kind::f16
 *                 MMAs; 2^-22 relative to each element: FP32-class, Q15).
 *                 1 = TF32X3 (x = hi + lo in tf32, 3 kind::tf32 MMAs).
 *                 3 = F16I8, opt-in only, NOT FP32-class: int8 codes
 *                 q = rint(x 2^e / 256), l = rint(8 h1); one kind::f16 MMA for
 *                 h0 h0' and one kind::i8 MMA for 32 (q l' + l q'); the error
 *                 is fixed point relative to the row maximum (~2^-18 of it,
 *                 normwise, not elementwise; Q15b); needs cta_group
 *                 2, b % 64 == 0 and K <= 131072 per update.
 *   "cta_group":  1 or 2 (default 2: CTA pairs, cta_group::2, 256-row tiles).
 *   "kernel_variant": -1 (auto, default: F16X3 / TF32X3 8, F16I8 6 -- 5 in
 *                 NCCL contexts, whose kernels need shared memory beside the
 *                 update) or 0..8, 12, 13, see fpm_k_update_f32.
 *   "chunk_k":    variants 7 / 8 / 12 / 13: K summed per TMEM accumulation before the
 *                 epilogue adds it to its FP32 register sum (0 = auto = 512;
 *                 DESIGN.md Q15c: the tensor cores' accumulation error grows
 *                 with the MMAs folded into one sum).
 *   "fuse":       pivots fused into one rank-(f b) update (FP32): 0 = auto
 *                 (f = min(8, max(1, 2048 / b))), else 1..8.  Groups never
 *                 straddle a column or row boundary of the arrangement, so a
 *                 group's exchange is its first pivot's plan with f-times longer
 *                 panels; the F16X3 scales are taken over the fused rows.  Halves
 *                 (f = 2) the C read-modify-write traffic of the iteration loop.
 *   "ooc_keep":   out-of-core devices (pmm_set_device_option "c_cap_bytes"):
 *                 1 (default) = P:34's refinement: the band order reverses
 *                 every other update and the last R bands of an update stay
 *                 on the device for the next one (the paper keeps two: R
 *                 transfers saved in each direction per update); 0 = every
 *                 band in and out every update.
 *   "ooc_buffers": R, out-of-core band buffers sharing the C cap, 2..16
 *                 (default 8; 2 = the paper's C0 / C1).  More, smaller bands
 *                 overlap the two copy directions with each other and with the
 *                 updates; with "ooc_keep" the per-update traffic stays C_i
 *                 minus the cap in each direction.  Fewer buffers (not below
 *                 2) are used when R bands of 256 rows exceed the cap.
 *   "graph":      1 (default): pmm_compute captures the whole k-loop (every
 *                 device's exchange, staging and update streams, forked from and
 *                 joined into device 0's compute stream) into one CUDA graph on
 *                 first use and replays it; timing events become event-record
 *                 nodes so per-group statistics are kept.  Re-captured after
 *                 pmm_setup, pmm_ipc_import or any option change.  NCCL
 *                 contexts, green partitions ("sm_partition" = 1: replays
 *                 were measured to lose the per-device SM confinement), pmm_run
 *                 and pmm_compute_into issue eagerly.
 *                 0: always eager.
 *   "e2e_tail":   update groups run band-major at the end of pmm_run /
 *                 pmm_compute_into so the copy of C_i to the host overlaps them
 *                 (FP32, resident C_i): -1 auto (default: enough groups to
 *                 cover the copy at ~55 GB/s), 0 off, 1..16.
 *   "tail_band":  rows of C_i per band of that tail, a positive multiple of
 *                 256 (default 2048); the last band's copy stays exposed.
 *   "tail_fuse":  1 (default; FP32 local / IPC contexts): the tail's pivots are
 *                 staged side by side as ONE operand with one F16X3 scale per
 *                 row / column over all of them (maxima merged first), so each
 *                 band takes a single update and one read-modify-write of C;
 *                 0: one update per tail group and band.
 *   "tail_stream": 1 (default): pmm_run on a context whose one device holds
 *                 the whole problem uploads the fused tail's B rows first and
 *                 its A rows band by band (a 4-byte-per-element staging buffer
 *                 of H x tail_K), staging and updating each band as it lands,
 *                 so the copy of C to the host overlaps the last uploads; the
 *                 tail may then be longer (the uploads under the groups before
 *                 it are 8 B per element for those groups + 4 B for the tail's
 *                 B).  When the host link is slower than the updates (upload
 *                 time per element of C_i >= half the k-loop's, e.g. N = 16384
 *                 on a full B200) the auto tail is the whole k-loop (up to 16
 *                 groups), so a step costs about its H2D bytes plus one band.
 *                 Same results bit for bit as 0 at the same tail length (all
 *                 tail pivots uploaded before the tail starts).
 *   "sm_partition": how an SM cap is enforced.  0 (default): the cap is the
 *                 grid of the persistent update kernel (one CTA per SM); other
 *                 kernels of the device are not confined, and devices sharing a
 *                 GPU may have caps summing above its SM count.  1: every device
 *                 gets a disjoint green-context partition of exactly its cap
 *                 (CUDA driver green contexts, SM-pair granularity, one split per
 *                 GPU) and all its kernels -- update, staging, NCCL -- run inside
 *                 it.  Needs a cap on every device and the caps of the devices
 *                 of one GPU to fit it (FPM_EUNSUPPORTED otherwise).  Rebuilds
 *                 the devices' streams: set it before pmm_setup.
 *   "share_b":    1 (default): in a local FP32 context, a device whose column's
 *                 B pivot owner is another device on the same GPU reads the
 *                 owner's staged (split, transposed) B operand instead of
 *                 staging its own copy (update groups outside the download
 *                 tail; the owner's next staging into that slot waits for
 *                 those updates); 0: every device stages its own.
 *   "fused_staging": 1 (default): FP32 F16X3 on the default update kernel --
 *                 update g's staging warp stages group g + 1 (the pivot pulls
 *                 from the holders' / owner's memory, the split, the B
 *                 transpose) while its MMAs run, instead of the standalone
 *                 staging kernels, which cannot run beside the persistent
 *                 update and so sat between two updates.  Applies to a GPU
 *                 device that is alone on its GPU in the context or confined
 *                 to its own green partition, in core, not in NCCL mode, whose
 *                 rectangle is large enough for the staging warps to finish
 *                 inside the update (DESIGN 4.8); under pmm_run the warps
 *                 first wait for the holders' upload-progress flags.  With
 *                 share_b a column member stages only its A rows.
 *                 Bit-identical C.  0: standalone staging kernels; 2: in-kernel
 *                 staging whatever the rectangle size.
 *   "sample_rel_ci_permille": fpm_sample's stop rule, the 95 % confidence
 *                 half-width in thousandths of the mean (default 25 = 2.5 %,
 *                 reading Q8; at most 50 repetitions either way).
 *   "raster_group": tile-rows per L2 raster group of the update (0 = auto,
 *                 the default: 12 for F16I8, 16 for F16X3 / TF32X3, measured
 *                 at c5, times the device's share of the SMs of its GPU among
 *                 the context's devices on it, at least 1: devices sharing a
 *                 GPU share its L2, so their A groups must fit it together).
 *   "l2_hint_b":  L2 policy of the B^T operand tiles: 0 normal (default),
 *                 1 evict-first, 2 evict-last.
 * FPM_EINVAL on unknown key or value. */
int pmm_set_option(pmm_ctx* ctx, const char* key, int64_t value);

/* Per-device knobs; `dev` is the device's index in the arrangement (must be
 * driven by this context).  Takes effect at the next pmm_setup.
 *   "c_cap_bytes": device memory C_i may occupy (0 = unlimited, default).
 *                  When the H x W C_i of a problem is larger, C_i is held OUT OF
 *                  CORE (PAPER.md P:34-40 GPU kernel versions 2-3): it
 *                  lives in pinned host memory and every update streams it
 *                  through a ring of R device band buffers (option
 *                  "ooc_buffers"; R = 2 is the paper's "C0 and C1") of
 *                  at most c_cap_bytes / R each (whole multiples of 256 rows,
 *                  at least 256), the host -> device copy of a later band and
 *                  the device -> host copy of an earlier one overlapping the
 *                  update of the current band on separate streams.  A_i, B_i
 *                  and the pivot buffers stay resident.
 *                  fpm_sample honours the cap (sizes whose C exceeds it are
 *                  timed out of core), so the speed function shows the memory
 *                  cliff that makes CPM fail (Table III).
 * FPM_EINVAL on unknown key / device or bad value. */
int pmm_set_device_option(pmm_ctx* ctx, int32_t dev, const char* key, int64_t value);

/* --------------------------------------- kernel-level entry points (tests)
 * Device pointers on the current CUDA device, launched asynchronously on
 * `stream` (a cudaStream_t; NULL = the legacy default stream). */

/* FP32 operand split of a rows x K panel (row stride ld, elements) for the
 * tensor cores (reading Q15).  scheme 0 (F16X3): hi/lo are fp16 rows x K,
 * inv_scale[rows] receives 2^-e of each row.  scheme 1 (TF32X3): hi/lo are
 * fp32 rows x K holding tf32 values; inv_scale unused (may be NULL).
 * scheme 3 (F16I8, Q15b): hi = fp16 h0 rows x K; lo = int8 codes, 2 K bytes
 * per row, one 128-byte row [q of 64 | l of 64] per 64-wide k-block (the
 * fpm_k_split_cols_f32 output is [l | q], so one int8 product of the two
 * gives both cross terms); K % 64 == 0.
 * K % 4 == 0, ld % 4 == 0. */
int fpm_k_split_f32(const float* src, int64_t ld, int64_t rows, int64_t K, int32_t scheme,
                    void* hi, void* lo, float* inv_scale, void* stream);

/* The same split applied to the transpose of a B pivot row: src is K x W
 * (row stride ld), hi/lo receive W x K (K-major), inv_scale[W] the per-column
 * scales of src.  One pass, no shared memory.  K % 8 == 0, W % 4 == 0. */
int fpm_k_split_cols_f32(const float* src, int64_t ld, int64_t K, int64_t W, int32_t scheme,
                         void* hi, void* lo, float* inv_scale, void* stream);

/* dst (cols x rows, contiguous) = transpose of src (rows x cols, row stride
 * ld); dt = FPM_F32 or FPM_F64.  Used for the K-major B pivot panel. */
int fpm_k_transpose(const void* src, int32_t dt, int64_t ld, int64_t rows, int64_t cols, void* dst,
                    void* stream);

/* Rank-b update C (M x Nc, row-major, ldc) += A (M x K) x B with B
 * given as Bt (Nc x K, K-major), operands as produced by fpm_k_split_f32 with
 * the same scheme (sa / sb: inverse row scales of A and Bt for F16X3, NULL
 * for TF32X3).  cta_group 1 or 2; num_sms = persistent grid (0 = all SMs).
 * accumulate = 0 writes C = A x B without reading C.  variant (cta_group 2):
 * shared-memory split between the operand ring and the C ring: 0 = 128-byte
 * k-blocks x 3 stages + 2 C chunks in flight, 1 = 64-byte x 4 + 6, 2 = 128-byte
 * x 2 + 6, 3 = 64-byte x 5 + 4, 4 = 128-byte x 2 + 4 (leaves ~36 KB smem per
 * SM for NCCL / staging kernels co-running with the update), 5 = 128-byte x 3
 * + 2 with C updated by TMA reduce-add (C never loaded into shared memory);
 * variants 0..5 sum a whole update in one TMEM accumulation.  7 =
 * chunked accumulation: every 512 of K is a fresh TMEM accumulation drained
 * into per-thread FP32 register sums (round-to-nearest), C written once per
 * tile by TMA reduce-add (store when accumulate = 0), 3 x 64-KB operand
 * stages; 8 = the same with 2 stages (160 KB).  12 / 13 (F16X3 only) =
 * variants 8 / 7 on clusters of two CTA pairs that share each B^T k-block by
 * TMA multicast (same C bit for bit; measured slower on B200).
 * -1 = auto (8).
 * scheme 3 (F16I8; cta_group 2, K % 64 == 0; sa / sb required): the
 * fp16 + int8 kernel, variants 0 = 2 x 64-KB stages + 4 C chunks,
 * 1 = 3 stages + 2 chunks, 2 = 2 + 6, 3 = 64-byte k-blocks x 5 + 4, 5 = variant
 * 0 and 6 = variant 1 with C updated by TMA reduce-add (the L2 adds the scaled
 * accumulator; C is never loaded into shared memory; 6 is the auto choice),
 * 4 = variant
 * 0 on clusters of two CTA pairs that multicast the B^T tiles (grid = the
 * co-resident clusters of 4); timing probes (C is not a product): 9 = no
 * operand loads and no C traffic (the MMAs and the TMEM drain only), 10 =
 * operand loads but no C traffic, 11 = C traffic but no operand loads.
 * scheme 2 is a timing probe (int8 operands, three kind::i8 MMAs per k-step,
 * s32 accumulator converted to float): it measures the int8 tensor path, its
 * result is not a product of FP32 operands.
 * Requires K % 8 == 0, ldc % 4 == 0. */
int fpm_k_update_f32(const void* a_hi, const void* a_lo, const void* bt_hi, const void* bt_lo,
                     const float* sa, const float* sb, float* C, int64_t M, int64_t Nc, int64_t K,
                     int64_t ldc, int32_t scheme, int32_t cta_group, int32_t num_sms,
                     int32_t accumulate, int32_t variant, void* stream);

/* Diagnostic counters of the F16I8 update's MMA issuer (the leader CTA of
 * each pair, lane 0; clock64 cycles summed over CTAs and launches): op 1 =
 * reset and enable for subsequent launches, 0 = disable, 2 = read into
 * out[4] = {cycles waiting for TMEM (the epilogue's drain of the previous tile),
 * cycles waiting for operands (TMA), cycles of the issuer loop, tiles}.
 * Current CUDA device; synchronise before reading. */
int fpm_k_prof(int32_t op, uint64_t* out);

/* Rank-b update in FP64 on DMMA: C (M x Nc, ldc) (+)= A (M x K, lda) x Bt^T,
 * Bt (Nc x K); accumulate = 0 overwrites C. */
int fpm_k_update_f64(const double* A, int64_t lda, const double* Bt, double* C, int64_t M, int64_t Nc,
                     int64_t K, int64_t ldc, int32_t accumulate, void* stream);

/* Fill a rows x cols window (ld elements) of the seeded global N x N matrix
 * starting at global (r0, c0); dt = FPM_F32 or FPM_F64; dist = fpm_dist. */
int fpm_k_fill_synthetic(void* dst, int32_t dt, int64_t ld, uint64_t seed, int64_t N, int64_t r0,
                         int64_t c0, int64_t rows, int64_t cols, int32_t dist, void* stream);

/* ---------------------------------------------------- host-CPU devices */

/* Host-CPU rank-b update kernel of the CPU devices (a
 * socket of c cores executing the GEMM kernel simultaneously; SURVEY §8(f)
 * NEXT-3), callable on its own: C (M x N, ldc) (+)= A (M x K) x B (K x N, ldb),
 * host pointers, row-major, dt = FPM_F32 (FP32 FMA arithmetic: SGEMM) or
 * FPM_F64.  A is read in K-segments of `seg` columns:
 * A(i, k) = A[(k / seg) * seg_stride + i * lda + k % seg] (seg = K,
 * seg_stride = 0 for a plain row-major A) -- the layout of a device's
 * block-column panels.  threads: worker threads (rows of C split evenly across
 * them), pinned to the first `threads` cores of this process's affinity mask
 * when pin != 0, else unpinned.  accumulate = 0 overwrites C.  Needs no GPU.
 * Errors: FPM_EINVAL (bad shape, threads < 1). */
int fpm_k_cpu_gemm(int32_t dt, int64_t M, int64_t N, int64_t K, const void* A, int64_t lda, int64_t seg,
                   int64_t seg_stride, const void* B, int64_t ldb, void* C, int64_t ldc, int32_t accumulate,
                   int32_t threads, int32_t pin);

/* Micro-kernel instruction set of the CPU GEMM on this host: writes
 * "avx512", "avx2" or "generic" (NUL-terminated, at most cap bytes). */
int fpm_cpu_isa(char* out, int32_t cap);

/* Host cores this process may use (its affinity mask), ascending: writes
 * min(count, cap) core ids to cores_out and the count to *count. */
int fpm_cpu_cores(int32_t* cores_out, int32_t cap, int32_t* count);

#ifdef __cplusplus
}
#endif

#endif /* FPMPMM_H */
