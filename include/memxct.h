/*
 * memxct.h -- C ABI of the B200-native MemXCT hot path.
 *
 * Paper: M. Hidayetoglu, T. Bicer, S. Garcia de Gonzalo, B. Ren, D. Gursoy, R. Kettimuthu,
 * I. Foster, W. Hwu, "MemXCT: Memory-Centric X-ray CT Reconstruction with Massive
 * Parallelization", SC'19.  "P:n" cites line n of the paper text (reference PAPER.md);
 * readings R1..R20 are listed in DESIGN.md section 3.
 *
 * Problem (eq. 1, with R = 0 and C = R^n): least squares  min_x ||y - A x||^2  where
 *   x  = tomogram, N x N pixels, natural index i*N + j, row i along +y;
 *   y  = sinogram, M projections x C channels, natural index m*C + k;
 *   A  = memoized ray-tracing matrix, A[r, p] = length of ray r inside pixel p, built once by
 *        Siddon tracing, parallel beam, theta_m = m*pi/M, unit-spaced centred
 *        channels (readings R1-R4).  A is stored once in fp32.
 *
 * Hot path: forward projection y = A x and backprojection x = A^T y as
 * gather-only SpMVs (Listing 2), rows and columns reordered by the
 * two-level pseudo-Hilbert ordering, inputs staged through a multi-stage shared-memory
 * buffer addressed with 16-bit indices (Listing 3), and CG iterations.
 *
 * Conventions
 *  * Ownership: a plan owns every device allocation it makes (matrices, maps, scratch, CG
 *    vectors, NCCL communicator).  Vector pointers passed in are caller-owned and never retained
 *    past the call.
 *  * Device vs host: memxct_forward/back/cg take DEVICE pointers (cudaMalloc / torch CUDA
 *    tensors) on the plan's device; the *_host variants take HOST pointers (pinned or pageable)
 *    and do the host<->device copies inside the call (stream-ordered, then synchronised).
 *  * dtype: float* (fp32) in PRECISION = FP32 mode, double* (fp64) in PRECISION = MIXED mode.
 *    The matrix values are fp32 in both modes.
 *  * Vector order: VECTOR_ORDER = 0 (default, P = 1 only): natural row-major tomogram [N][N] and
 *    sinogram [M][C].  VECTOR_ORDER = 1: the plan's local Hilbert order (see
 *    memxct_local_indices); required when P > 1.
 *  * Asynchrony: forward, back and cg are stream-ordered on `cuda_stream` (a cudaStream_t; NULL =
 *    legacy default stream).  build is synchronous.  cg synchronises only when residual_norms is
 *    non-NULL (it copies the norms to the host).
 *  * Errors: every call returns a status; no C++ exception crosses the ABI.  The detail of the last
 *    error on the calling thread is memxct_last_error().  After MEMXCT_ERR_OUT_OF_MEMORY the plan
 *    stays valid for memxct_plan_destroy.
 *  * No CPU fallback: every arithmetic step runs in this library's CUDA kernels; without a CUDA
 *    device memxct_build returns MEMXCT_ERR_CUDA.
 */
#ifndef MEMXCT_H
#define MEMXCT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MEMXCT_VERSION_MAJOR 0
#define MEMXCT_VERSION_MINOR 1

typedef struct memxct_plan* memxct_plan_t; /* opaque */

typedef enum {
    MEMXCT_OK = 0,
    MEMXCT_ERR_INVALID_ARG = 1,  /* bad size, null pointer, option out of range */
    MEMXCT_ERR_STATE = 2,        /* plan used before build, option set after build, ... */
    MEMXCT_ERR_OUT_OF_MEMORY = 3,/* device or host allocation failed */
    MEMXCT_ERR_CUDA = 4,         /* CUDA runtime / launch error, or no device */
    MEMXCT_ERR_NCCL = 5,         /* P > 1 communication error: an NCCL error (including an
                                  * asynchronous one, polled with ncclCommGetAsyncError at every call
                                  * on a decomposed plan), or a fused-exchange wait on the device
                                  * that timed out (~20 s: a peer is gone; reported at the next call,
                                  * the interrupted call's results are undefined) */
    MEMXCT_ERR_UNSUPPORTED = 6   /* valid request this build does not implement */
} memxct_status_t;

typedef enum {
    /* Tile side of the first Hilbert level (power of two, 1..128).  Default (reading R7):
     * largest power of two T with 8T <= min(H, W), clamped to [4, 64]. */
    MEMXCT_OPT_TILE_TOMO = 0,
    MEMXCT_OPT_TILE_SINO = 1,
    /* Rows per partition (one CTA per partition; one 32-row slice per warp).
     * Multiple of 32 in [32, 1024] used for both directions, or 0 = auto (default), chosen per
     * direction: the largest multiple of 32 in [128, 1024] whose partition count spreads over the
     * SMs with <= 3 % wave-quantisation loss (layout.cu: resolve_tuning).  get_option returns
     * the forward value after build; memxct_layout_info reports both. */
    MEMXCT_OPT_PART_ROWS = 2,
    /* Stage-buffer capacity in fp32 entries (16-bit local addressing).
     * 256 <= value <= 57344 (224 KB), or 0 = auto (default, per direction): 36 * R.  MIXED mode stages
     * value/2 fp64 entries in the same bytes. */
    MEMXCT_OPT_BUFFER_ENTRIES = 3,
    /* 0 = FP32 (fp32 vectors, fp32 FMA; the paper's precision), 1 = MIXED (fp32 A, fp64
     * vectors and fp64 FMA).  Default 0. */
    MEMXCT_OPT_PRECISION = 4,
    /* 1 = canonical summation order (reading R16): one fp64 fma chain per row in ascending
     * Hilbert column order, dots as per-partition fma chains summed in partition order.
     * Requires PRECISION = MIXED.  Single GPU only (P = 1): at P > 1 a row's sum is split
     * over the ranks that own its pixels (A = R C A_p), so one chain per row does not
     * exist; memxct_build on a decomposed plan gives MEMXCT_ERR_UNSUPPORTED.  Default 0. */
    MEMXCT_OPT_CANONICAL = 5,
    /* 0 = recursive-residual CGLS (default, 1 forward + 1 back per iteration, reading R13).
     * 1 = explicit residual r = y - A x each iteration (2 forward + 1 back). */
    MEMXCT_OPT_CG_VARIANT = 6,
    /* 0 = natural row-major vectors (default, P = 1 only); 1 = plan (local Hilbert) order. */
    MEMXCT_OPT_VECTOR_ORDER = 7,
    /* 1..8: slices per matrix stream the batched calls are tuned for (multi-slice reconstruction,
     * P:943-947).  The automatic stage buffer becomes 36 * PART_ROWS / 2^ceil(log2(SLICES))
     * entries so that many slices' inputs fit in shared memory, and (FP32) the entries of every
     * row are stored in a shared-memory-bank-aware order instead of ascending input order (same
     * sums up to fp32 rounding order).  Default 1. */
    MEMXCT_OPT_SLICES = 8,
    /* P > 1 exchange: 0 = grouped ncclSend/ncclRecv all-to-allv between the SpMV and
     * the reduction (default); 1 = fused over peer memory (FP32, P <= 16): the SpMV epilogue
     * stores partials straight into the owners' receive buffers and the owners' pack kernel stores
     * ray values straight into the peers' footprint buffers (CUDA IPC mappings over NVLink),
     * synchronised by epoch/credit flags -- no separate collective on the data path; the CG dots
     * go over peer memory too.  2 = dense collectives (the comparison of SURVEY 8(e)): forward
     * partials scattered into a zeroed P x max-owned-range sinogram and ncclReduceScatter, back
     * ncclAllGather of the owned values and a gather of the footprint rays -- more bytes moved
     * (the whole sinogram instead of the ~0.4 M C interacting rays), no per-peer bookkeeping. */
    MEMXCT_OPT_EXCHANGE = 9,
    /* Row grouping of the forward SpMV's partitions (A_p rows = rays).  -1 = the paper's: a
     * partition is PART_ROWS consecutive rays in Hilbert order (a square of about
     * sqrt(R) x sqrt(R) projections x channels).  a > 0 (power of two <= PART_ROWS / 32): rays are
     * grouped into blocks of `a` consecutive projections x PART_ROWS / a consecutive channels
     * (projection-major, channel-minor inside a block) before being cut into partitions, which
     * raises the stage-buffer reuse when consecutive projections are many pixels apart (few
     * projections, wide detector: config 5).  0 = auto (default): blocks with a = the smallest
     * power of two >= 2 a*, a* = sqrt(R / (L pi / M)), L = side of the local tomogram (measured
     * optimum for whole tomograms and for rank regions), when a* <= sqrt(R)/4, else -1.
     * A rank's blocks count channels from the channel of its region's centre at each projection,
     * so a block's rays cross inside the region.  Vector layouts and results are unchanged: each row still sums its entries in
     * ascending Hilbert input order (FP32 outputs bit-identical).  CANONICAL forces -1. */
    MEMXCT_OPT_RAY_BLOCK = 10,
    /* Stage order of the forward SpMV (A_p): -1 = the paper's (reading R10): a partition's
     * distinct input pixels sorted by Hilbert index and cut into stages of BUFFER_ENTRIES.
     * 1 = slab order: sorted by (band of 16 pixels across the direction of the partition's rays,
     * then Hilbert index), so every stage is a band that all of the partition's rays cross and all
     * warps have work in every stage.  Same map entries and bytes; each
     * row sums the same products in another order (FP32 results equal up to rounding).  0 = auto
     * (default): slab order in FP32 mode; -1 in MIXED mode, whose fp64 row chains then ascend in
     * Hilbert order like the oracle's canonical sums.  CANONICAL forces -1. */
    MEMXCT_OPT_STAGE_ORDER = 11
} memxct_option_t;

/* Create a plan for an N x N tomogram and an M x C sinogram.  Host only; no device
 * work.  n, projections, channels must be >= 1 and n*n, projections*channels < 2^31. */
memxct_status_t memxct_plan_create(int32_t n, int32_t projections, int32_t channels,
                                   memxct_plan_t* out);

/* Set a tuning/precision option (table above) before memxct_build; ERR_STATE afterwards. */
memxct_status_t memxct_plan_set_option(memxct_plan_t plan, memxct_option_t option, int64_t value);
memxct_status_t memxct_plan_get_option(memxct_plan_t plan, memxct_option_t option, int64_t* value);

/* Multi-GPU (P > 1, A = R C A_p): rank in [0, nranks), a 128-byte ncclUniqueId
 * produced by rank 0 and broadcast by the caller, and the CUDA device of this rank.  Before
 * build.  With nranks == 1: a NULL id means the plain single-GPU plan; a non-NULL id runs the
 * decomposed path (footprint, exchange maps, NCCL send/recv and allreduce) on a one-rank
 * communicator -- same results, used to exercise the multi-GPU code on one device. */
memxct_status_t memxct_plan_set_comm(memxct_plan_t plan, int32_t rank, int32_t nranks,
                                     const void* nccl_unique_id, int32_t cuda_device);

/* Fill a 128-byte buffer with a fresh ncclUniqueId (call on rank 0 only).  NCCL is loaded at
 * run time (dlopen of libnccl.so.2); MEMXCT_ERR_NCCL if it is unavailable. */
memxct_status_t memxct_get_unique_id(void* nccl_unique_id_out);

/* Virtual ranks (testing the multi-GPU path on one device): a group of `nranks` plans in one
 * process, each built and driven from its own host thread, whose collectives are device copies
 * instead of NCCL.  Same decomposition, maps, kernels and results as NCCL ranks; not graph
 * captured.  The group must outlive its plans. */
typedef struct memxct_group* memxct_group_t;
memxct_status_t memxct_local_group_create(int32_t nranks, memxct_group_t* out);
memxct_status_t memxct_local_group_destroy(memxct_group_t group);
memxct_status_t memxct_plan_set_comm_local(memxct_plan_t plan, memxct_group_t group, int32_t rank);

/* Host transport (processes of one node, possibly sharing one GPU): rank in [0, nranks <= 16) of
 * a job whose processes rendezvous through the POSIX shared-memory segment `name` ("/<token>",
 * unique per job and plan; rank 0 creates it at build, the others attach, rank 0 unlinks it once
 * all are attached -- the caller broadcasts the name, e.g. over torch.distributed gloo).  The
 * build's collectives and the collective exchanges (EXCHANGE = 0, 2) move device data between the
 * processes through CUDA-IPC-mapped device mailboxes with host barriers; the fused exchange
 * (EXCHANGE = 1) maps the peers' buffers with cudaIpcOpenMemHandle and synchronises through
 * system-scope flags exactly as NCCL ranks do (waits in one-thread kernels when the ranks share a
 * GPU).  Same decomposition, kernels and results as NCCL ranks / virtual ranks (sums over ranks in
 * rank order); not graph-captured.  The multi-process form of the virtual ranks: it runs the
 * cross-process data plane where NCCL cannot (NCCL rejects two ranks on one device).  Before
 * build.  Errors: INVALID_ARG (rank, name), NCCL (a peer process never arrives: ~300 s). */
memxct_status_t memxct_plan_set_comm_host(memxct_plan_t plan, int32_t rank, int32_t nranks,
                                          const char* name, int32_t cuda_device);

/* Host-only round trip of the host transport (no device needed): rendezvous on `name` (as in
 * memxct_plan_set_comm_host), a host allgather of one int64 per rank into gathered[0..nranks)
 * (host), a barrier, teardown.  For checking the processes' rendezvous (e.g. the CPU gloo tests).
 * The rendezvous gives up after MEMXCT_HOST_COMM_TIMEOUT_S seconds (default 300): NCCL status. */
memxct_status_t memxct_host_comm_probe(const char* name, int32_t rank, int32_t nranks, int64_t value,
                                       int64_t* gathered);

/* Shard probe: build on this device only rank `rank`'s part of a `nranks`-way decomposition
 * -- the same tile ranges (R12), footprint rays, A_p, A_p^T and exchange counts /
 * maps that rank would build inside a real P-rank job, with no peers and no communicator (the
 * build's collective steps are replaced by tracing every ray locally).  It answers "what does
 * one of P GPUs hold and how fast are its kernels" for decompositions whose other ranks do not
 * fit or do not exist (config 5's 11293^2 slice, ~43 GB of A_p per rank at P = 8).  Before
 * build.  After build: memxct_footprint_*, memxct_spmv_time, memxct_exchange_info / _counts,
 * memxct_domain_ranges, memxct_local_size / _indices, memxct_stats and memxct_layout_info work;
 * the whole operators (forward, back, cg, sirt, batched and host variants, exchange_time) return
 * MEMXCT_ERR_UNSUPPORTED, as does EXCHANGE = 1 at build. */
memxct_status_t memxct_plan_set_shard(memxct_plan_t plan, int32_t rank, int32_t nranks,
                                      int32_t cuda_device);

/* Domain decomposition helper (host only, reading R12): split `count` tiles with
 * nonnegative `weights` (nonzeros per tile, in Hilbert order) into `parts` contiguous ranges
 * with about equal weight; bounds[0..parts] (host) receives the range boundaries, every range
 * non-empty when count >= parts.  memxct_build uses it for both domains. */
memxct_status_t memxct_partition_ranges(const int64_t* weights, int64_t count, int32_t parts,
                                        int64_t* bounds);

/* After build: the Hilbert-index ranges owned by every rank (bounds[0..nranks]) for domain 0
 * (tomogram pixels) or 1 (sinogram rays). */
memxct_status_t memxct_domain_ranges(memxct_plan_t plan, int32_t domain, int64_t* bounds);

/* After build (P > 1): this rank's footprint rays (rows of A_p), the partial-sinogram entries it
 * sends per forward exchange and receives (the back exchange is the reverse), and the number of
 * peers it talks to.  Any pointer may be NULL. */
memxct_status_t memxct_exchange_info(memxct_plan_t plan, int64_t* footprint_rays,
                                     int64_t* sent_entries, int64_t* received_entries,
                                     int32_t* peers);

/* After build, decomposed plans only (set_comm with an id, set_comm_local, set_shard; else
 * INVALID_ARG): send_counts[q] / recv_counts[q] (host, nranks int64 each, nullable) = partial-sinogram
 * entries this rank sends to / receives from rank q per forward exchange (q = rank: its own slice). */
memxct_status_t memxct_exchange_counts(memxct_plan_t plan, int64_t* send_counts, int64_t* recv_counts);

/* The local operator A_p of P:758-761 alone, decomposed plans only.  Rows of A_p are this rank's
 * footprint rays: every ray with a segment in its pixels, in Hilbert order (owner, Hilbert).
 * memxct_footprint_rays writes their natural indices (host, footprint_rays int64, see
 * memxct_exchange_info).  memxct_footprint_forward: y_footprint[i] = sum over LOCAL pixels p of
 * A[ray_i, p] x_local[p] (x_local in plan order, local_size(0) entries; y_footprint:
 * footprint_rays entries) -- the partial projection before exchange and reduction.
 * memxct_footprint_back: x_local = A_p^T y_footprint.  Device pointers, dtype per PRECISION,
 * stream-ordered, outputs overwritten. */
memxct_status_t memxct_footprint_rays(memxct_plan_t plan, int64_t* natural_ray);
memxct_status_t memxct_footprint_forward(memxct_plan_t plan, const void* x_local, void* y_footprint,
                                         void* cuda_stream);
memxct_status_t memxct_footprint_back(memxct_plan_t plan, const void* y_footprint, void* x_local,
                                      void* cuda_stream);

/* Preprocessing: Hilbert ordering and domain decomposition, Siddon tracing of A on
 * the device, order-preserving transposition to A^T, partitioning and the multi-stage buffered
 * layout of both matrices.  Synchronous; collective over the communicator when P > 1.
 * `cuda_stream` may be NULL. */
memxct_status_t memxct_build(memxct_plan_t plan, void* cuda_stream);

/* Per-phase wall-clock seconds of the last memxct_build (preprocessing throughput, SURVEY 8(f)
 * NEXT-3; the paper's preprocessing, timed at 4.00 s for ADS2 and 139 s for RDS1 per
 * KNL node).  `seconds` (host) receives MEMXCT_BUILD_PHASES doubles, in
 * this order:
 *   0 hilbert     two-level pseudo-Hilbert permutations of both domains
 *   1 decompose   domain decomposition: column-count histogram + tile ranges (P > 1)
 *   2 count       Siddon count pass of every ray (row lengths; footprint at P > 1)
 *   3 trace_fwd   Siddon emit pass of A / A_p
 *   4 sort_fwd    per-row ordering of A's entries (segmented sort; slab order)
 *   5 layout_fwd  partitions, stage cut, 16-bit SELL layout of A, row grouping
 *   6 trace_back  pixel histogram + count + emit passes of the transposition's chunks
 *   7 transpose   order-preserving stable radix sort by pixel
 *   8 layout_back partitions, stage cut, layout of A^T
 *   9 exchange    exchange maps (P > 1)
 *  10 total       the whole memxct_build call
 * Phases are separated by synchronisations the build performs anyway (CUDA events inside the
 * chunk loops), so they add up to the total up to host bookkeeping.  STATE before build. */
#define MEMXCT_BUILD_PHASES 11
memxct_status_t memxct_build_phases(memxct_plan_t plan, double* seconds);

/* Number of locally owned entries of a domain (0 = tomogram pixels, 1 = sinogram rays) and
 * their natural indices in plan order (host array of `count` int64).  At P = 1 the plan order is
 * the two-level pseudo-Hilbert order, i.e. natural_idx[h] = natural index of Hilbert position h. */
memxct_status_t memxct_local_size(memxct_plan_t plan, int32_t domain, int64_t* count);
memxct_status_t memxct_local_indices(memxct_plan_t plan, int32_t domain, int64_t* natural_idx);

/* Forward projection y = A x.  x: device tomogram (local_size(0) entries), y: device
 * sinogram (local_size(1) entries), dtype per PRECISION.  Overwrites y. */
memxct_status_t memxct_forward(memxct_plan_t plan, const void* x_tomo, void* y_sino,
                               void* cuda_stream);

/* Backprojection x = A^T y (a gather with the transposed matrix, no
 * atomics).  Overwrites x. */
memxct_status_t memxct_back(memxct_plan_t plan, const void* y_sino, void* x_tomo,
                            void* cuda_stream);

/* CGLS reconstruction (reading R13): x_0 = 0, exactly `iters` iterations (R14),
 * x_tomo overwritten.  residual_norms (host, iters + 1 doubles, nullable) receives ||r_k||
 * (R15); iterations skipped after gamma or delta reach 0 repeat the last norm.  iters == 0
 * writes zeros.  iters < 0 is INVALID_ARG. */
memxct_status_t memxct_cg(memxct_plan_t plan, const void* y_sino, void* x_tomo, int32_t iters,
                          double* residual_norms, void* cuda_stream);

/* SIRT on the same operators (the paper's comparison solver, 45 iterations,
 * P:907-912): x_0 = 0, x_{k+1} = x_k + C A^T R (y - A x_k) with R = 1 / row sums of A and
 * C = 1 / column sums (0 where a sum is 0).  residual_norms (host, iters + 1, nullable) receives
 * ||y - A x_k||, k = 0..iters.  Synchronous.  Same dtypes and vector order as memxct_cg. */
memxct_status_t memxct_sirt(memxct_plan_t plan, const void* y_sino, void* x_tomo, int32_t iters,
                            double* residual_norms, void* cuda_stream);

/* Collective (P > 1): device time, in microseconds, of one forward exchange (all-to-allv of the
 * partial sinograms + reduction R) and one back exchange (duplication R^T + reverse
 * all-to-allv), averaged over `reps` back-to-back repetitions timed with CUDA events on
 * `cuda_stream`.  Writes 0 at P = 1. */
memxct_status_t memxct_exchange_time(memxct_plan_t plan, int32_t reps, double* us_forward,
                                     double* us_back, void* cuda_stream);

/* Local, not collective: device time, in microseconds, of this rank's forward SpMV (A_p, or A
 * at P = 1) and back SpMV (A_p^T / A^T) kernels alone, without exchange, averaged over `reps`
 * back-to-back launches per direction (CUDA events on `cuda_stream`; zero-valued scratch inputs,
 * the access pattern does not depend on values).  Synchronous.  reps < 0: INVALID_ARG. */
memxct_status_t memxct_spmv_time(memxct_plan_t plan, int32_t reps, double* us_forward,
                                 double* us_back, void* cuda_stream);

/* Plan-independent probe of the roofline denominator: the achievable HBM read bandwidth of the
 * current device, in GB/s (1e9 B/s).  Allocates `bytes` (rounded down to 16 B; >= 16) of
 * device scratch, zeroes it, and streams it `reps` times (>= 1) with the SpMV's own 16 B
 * read-only, L1-bypassing, L2-evict-first load, grid-stride interleaved over all SMs, for three
 * launch shapes; writes the best average (CUDA events on `cuda_stream`).  Synchronous.  The
 * driver's MEASURED_PEAKS.json figure is a read+write copy, which a read-only stream (the
 * SpMV's matrix) may exceed; this gives the read-only ceiling beside it.  Errors: INVALID_ARG
 * (sizes, NULL gbs), OUT_OF_MEMORY, CUDA. */
memxct_status_t memxct_read_ceiling(int64_t bytes, int32_t reps, double* gbs, void* cuda_stream);

/* Multi-slice variants (the paper reuses the memoized matrices for every
 * slice): `slices` independent slices with the same geometry, vectors slice-major
 * (x[s * local_size(0) + i], y[s * local_size(1) + r]), FP32 only.  The slices are processed in
 * groups of up to 8 that share one stream of the matrix from HBM (an SpMM), each slice's
 * arithmetic identical to the single-slice call (bit-identical results).  memxct_cg_batch runs
 * `slices` (<= 32) independent CGLS solves; residual_norms (nullable) is [slices][iters + 1]. */
memxct_status_t memxct_forward_batch(memxct_plan_t plan, int32_t slices, const void* x_tomo,
                                     void* y_sino, void* cuda_stream);
memxct_status_t memxct_back_batch(memxct_plan_t plan, int32_t slices, const void* y_sino,
                                  void* x_tomo, void* cuda_stream);
memxct_status_t memxct_cg_batch(memxct_plan_t plan, int32_t slices, const void* y_sino,
                                void* x_tomo, int32_t iters, double* residual_norms,
                                void* cuda_stream);

/* Host-buffer variants: same semantics, HOST pointers; the H2D copy of the input, the device
 * computation and the D2H copy of the result all happen inside the call, which returns after
 * the result is on the host. */
memxct_status_t memxct_forward_host(memxct_plan_t plan, const void* x_host, void* y_host,
                                    void* cuda_stream);
memxct_status_t memxct_back_host(memxct_plan_t plan, const void* y_host, void* x_host,
                                 void* cuda_stream);
memxct_status_t memxct_cg_host(memxct_plan_t plan, const void* y_host, void* x_host,
                               int32_t iters, double* residual_norms, void* cuda_stream);

/* Byte model for the bench: nonzeros of A (= of A^T), stored SELL slots of both
 * directions, stage-map entries of both directions, device bytes held by the plan. */
memxct_status_t memxct_stats(memxct_plan_t plan, int64_t* nnz, int64_t* stored_slots,
                             int64_t* map_entries, int64_t* device_bytes);

/* Per-direction layout sizes (dir 0 = A / forward, 1 = A^T / back): partitions, total stages,
 * stored slots, map entries, rows, nonzeros, rows per partition (CTA) and stage-buffer entries
 * (fp64 entries in MIXED mode).  The automatic tuning picks R and B per direction.  Any pointer
 * may be NULL. */
memxct_status_t memxct_layout_info(memxct_plan_t plan, int32_t dir, int64_t* parts,
                                   int64_t* stages, int64_t* slots, int64_t* map_entries,
                                   int64_t* rows, int64_t* nnz, int64_t* part_rows,
                                   int64_t* buffer_entries);

/* Device-side export of the memoized matrix of direction `dir` (0 = A_p, 1 = A_p^T) as
 * unsorted COO, one entry per stored slot: `rows`, `cols`, `vals` are caller-owned DEVICE
 * arrays of memxct_layout_info's `slots` entries.  Entry = (output index, input index, value) in
 * the plan's vector order (natural indices with VECTOR_ORDER = 0); padding slots are written as
 * (-1, -1, 0).  Stream-ordered on `cuda_stream`.  For interoperability -- e.g. handing the same
 * matrix to another SpMV implementation -- not part of the hot path.
 * Errors: STATE before build, INVALID_ARG for dir or NULL arrays. */
memxct_status_t memxct_export_coo(memxct_plan_t plan, int32_t dir, int32_t* rows, int32_t* cols,
                                  float* vals, void* cuda_stream);

/* Copy the layout of partitions [p0, p1) of direction `dir` to host arrays (introspection for
 * tests; the layout is documented in DESIGN.md section 5):
 *   stage_base  int64[p1-p0+1]   global stage index range of each partition
 *   map_off     int64[p1-p0+1]   offset of each partition's map entries
 *   map         int32[...]       input index (plan order) of each stage-buffer slot
 *   slot_off    int64[(stages)*slices_per_part + 1]  slot offset of each (stage, slice) block
 *   ind         uint16[...]      local buffer index of each slot
 *   val         float[...]       value of each slot (0 for padding)
 *   lane_chunks uint16[(n_slot_off-1)*32]  8-slot chunks of each lane of each block
 *   part_row0   int64[p1-p0+1]   first row of each partition (R rows each, or equal-work
 *                                partitions of <= R rows under the automatic tuning)
 * Pass NULL for all arrays to query sizes through the int64 out-parameters. */
memxct_status_t memxct_layout_export(memxct_plan_t plan, int32_t dir, int64_t p0, int64_t p1,
                                     int64_t* stage_base, int64_t* map_off, int32_t* map,
                                     int64_t* slot_off, uint16_t* ind, float* val,
                                     uint16_t* lane_chunks, int64_t* part_row0, int64_t* n_map,
                                     int64_t* n_slot_off, int64_t* n_slots);

/* Output position of every layout row (dir 0: rows of A / A_p, dir 1: rows of A^T / A_p^T), host
 * array of layout_info rows int64: the index the row's result is written to in the call's output
 * vector -- natural (VECTOR_ORDER = 0), plan / Hilbert order (1) or footprint position (A_p of a
 * decomposed plan).  Identity unless the rows were regrouped (RAY_BLOCK) or the plan writes
 * natural order. */
memxct_status_t memxct_layout_rows(memxct_plan_t plan, int32_t dir, int64_t* out_index);

/* Destroy a plan and free everything it owns.  NULL-safe. */
memxct_status_t memxct_plan_destroy(memxct_plan_t plan);

const char* memxct_status_string(memxct_status_t status);
/* Detail of the last error on the calling thread ("" if none). */
const char* memxct_last_error(void);

/* Number of CUDA kernels this library has launched in this process (instrumentation for the
 * bench's gpu_launches claim; graph launches count every kernel node). */
int64_t memxct_kernel_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* MEMXCT_H */
