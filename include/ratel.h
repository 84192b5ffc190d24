/*
 * ratel.h -- C ABI of the B200-native active-gradient-offloading optimizer step.
 *
 * What the library does (PAPER.md = /root/reference/PAPER.md, "P:Lnnn"):
 *   Ratel's "active gradient offloading" (AGO, §IV-C) runs the
 *   optimizer handler for a transformer block as soon as that block's 16-bit
 *   gradient G16 arrives, "with a decreasing index during the backward stage"
 *   (P:L1038-1041), instead of as a separate stage after backward (the
 *   ZeRO-Infinity schedule).  The handler updates the
 *   fp32 master weights P32 and the Adam states OS32 (m, v) and "produces a
 *   16-bit parameter copy" P16 (sizes Table II);
 *   the paper runs it as a CPU Adam.  Here the
 *   handler is a fused sm_100a AdamW kernel launched on a dedicated optimizer
 *   stream ordered after the backward stream by a CUDA event, with the states
 *   either resident in HBM or held in pinned host memory and streamed through
 *   a ring of device tiles (the paper's Fig. 3b pipeline, with
 *   the host link in place of the SSD link).  AGO "keeps synchronous model
 *   updating" (footnote 4 P:L1147-1152): the result is
 *   identical to one synchronous Adam(W) step applied after backward.
 *
 * Update rule (the paper never writes it; it cites Adam [44], and
 * shows torch.optim.Adam(), Fig. 4).  DESIGN.md readings:
 *   g = fp32(G16) [* clip coef]
 *   RATEL_ADAMW  : theta *= (1 - lr*wd)          (decoupled decay, default)
 *   RATEL_ADAM_L2: g += wd*theta                 (torch.optim.Adam's decay)
 *   m = b1*m + (1-b1)*g ; v = b2*v + (1-b2)*g^2
 *   theta -= lr/(1-b1^t) * m / (sqrt(v)/sqrt(1-b2^t) + eps)
 *   P16 = bf16_rne(theta)  (from the stored fp32 master)
 * fp32 math (explicit FMA placement; sqrt and 1/denominator by the <= 1-ulp
 * sqrt.approx.f32 / rcp.approx.f32, reading R7 -- the IEEE forms are
 * the build flag RATEL_K1_FASTMATH=0; never --use_fast_math).
 *
 * Call protocol (one host thread per process, one process per GPU; not
 * re-entrant):
 *   ratel_init -> ratel_register_block* ->
 *     { ratel_adam_step(t) and ratel_offload_grad_chunk(b) for EVERY
 *       registered b, in any interleaving -> ratel_sync }* -> ratel_finalize
 *   A block's update is enqueued by whichever of ratel_adam_step(t) and its
 *   ratel_offload_grad_chunk() arrives second: arming before backward gives
 *   the paper's overlapped AGO, arming after all hand-offs gives the
 *   "Ratel+ZeRO" deferred baseline.  With max_grad_norm > 0
 *   every update waits for the last hand-off of the step (global norm).
 *
 * Ownership: every pointer registered is BORROWED (allocated by the caller,
 * e.g. torch) and must stay valid and unmoved until ratel_finalize.  Between
 * a block's hand-off and ratel_sync the caller must not touch that block's
 * master/exp_avg/exp_avg_sq/param nor overwrite its grad (in torch:
 * grad.record_stream(ratel_optimizer_stream()); such tensors must be
 * released before ratel_finalize destroys that stream).  The library owns only what
 * it creates: streams, events, device tiles, reduction buffers, NCCL comm.
 *
 * CUDA graphs: the step is not graph-capturable (the library tracks its tile
 * scheduler, arming state and collectives per call on the host); a stream
 * passed to ratel_offload_grad_chunk / ratel_block_wait / ratel_sync while it
 * is being captured is refused with RATEL_EINVAL before anything is enqueued.
 *
 * Errors: every int-returning call returns RATEL_OK (0) or a negative code.
 * RATEL_EINVAL / RATEL_ESTATE have no side effects.  A CUDA or NCCL failure
 * (including an asynchronous one detected later) is STICKY: every later call
 * returns it until ratel_finalize.  ratel_last_error() gives a thread-local
 * message for the last failure.
 */
#ifndef RATEL_H
#define RATEL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RATEL_ABI_VERSION 2   /* 2: ratel_config gained ssd_schedule and ssd_io (72 bytes) */
#define RATEL_MAX_BLOCKS 4096          /* block ids are 0 .. RATEL_MAX_BLOCKS-1 */
#define RATEL_MAX_RANGES_PER_BLOCK 32

enum {
  RATEL_OK = 0,
  RATEL_EINVAL = -1,     /* bad argument (pointer kind, alignment, size, value) */
  RATEL_ESTATE = -2,     /* call out of protocol order */
  RATEL_ECUDA = -3,      /* CUDA runtime failure (sticky) */
  RATEL_ENCCL = -4,      /* NCCL failure (sticky) */
  RATEL_ENOMEM = -5,     /* device/host allocation failed (sticky) */
  RATEL_ENONFINITE = -6, /* clip mode: global grad norm was NaN/Inf (update still applied, like torch) */
  RATEL_EIO = -7         /* SSD residency: a state file read/write failed (sticky) */
};

/* Where a block's fp32 states live and who updates them:
 *   DEVICE        states in HBM, the fused GPU kernel updates them in place;
 *   PINNED_HOST   states in page-locked host memory, streamed H2D/D2H through
 *                 a ring of device tiles around the same GPU kernel (the
 *                 paper's Fig. 3b pipeline with the host link as the link);
 *   HOST_COMPUTE  the paper's own design (§IV-C; CPU optimizer
 *                 P:L582-584): states in page-locked host memory, G16 copied
 *                 device->host (2 B/param), the CPU updates the states and
 *                 produces P16 (fp32 arithmetic, SIMD + OpenMP), P16 copied
 *                 host->device (2 B/param); stream-ordered via
 *                 cudaLaunchHostFunc, the host thread never blocks. */
/*   SSD           the paper's storage tier (§IV-C Fig. 3b; Eq. 5
 *                 "14P/BW_S2M + 14P/BW_M2S"): states in a file
 *                 (ratel_register_ssd); a reader thread streams each tile
 *                 file -> pinned staging -> device tile, the GPU kernel
 *                 updates it, and a writer thread writes it back, so the read
 *                 of tile k+1, the update of tile k and the write-back of
 *                 tile k-1 overlap.  A block's reads start when its gradient
 *                 is complete (the active message; the reader thread waits on
 *                 the hand-off event).  Single rank (no NCCL communicator). */
/*   Hybrid (both host resources at once): register the head of a range as a
 *                 PINNED_HOST block and the rest (a 16-byte-aligned split, the
 *                 five pointers offset by the split) as a HOST_COMPUTE block,
 *                 and hand both off together -- the host link and the host's
 *                 cores then update one block concurrently (DESIGN.md §7,
 *                 5.6-6.1 G params/s vs 4.0 / 5.1-5.3 for either alone). */
/*   SSD_HOST_COMPUTE  the paper's full pipeline (Fig. 3b with its CPU
 *                 optimizer): states in a state file exactly as RATEL_SSD
 *                 (ratel_register_ssd), but no state crosses the host link --
 *                 the reader thread copies the block's G16 device->host
 *                 (2 B/param), reads each tile file -> pinned staging, runs the
 *                 CPU AdamW on it (the HOST_COMPUTE handler) and queues it for
 *                 the writer thread; the P16 goes host->device (2 B/param).
 *                 Bitwise equal to HOST_COMPUTE.  Single rank. */
typedef enum { RATEL_DEVICE = 0, RATEL_PINNED_HOST = 1, RATEL_HOST_COMPUTE = 2, RATEL_SSD = 3,
               RATEL_SSD_HOST_COMPUTE = 4 } ratel_residency;
typedef enum { RATEL_ADAMW = 0, RATEL_ADAM_L2 = 1 } ratel_mode;
/* Pinned-host staging schedule: PIPELINED = Fig. 3b (stage-in of tile k+1,
 * update of tile k and write-back of tile k-1 overlap on three streams; the
 * tile updates run on a high-priority stream so they slot in between
 * backward kernels);
 * SERIALIZED = Fig. 3a (naive AGO: stage-in, update, write-back in series);
 * ZERO_COPY = no tiles: the register-staged update kernel (RATEL_UPDATE_LDG_LITE)
 * reads and writes the page-locked states in place over the host link
 * (unified addressing), one kernel per range; grid = cfg.max_ctas if set.
 * Results are identical in all three. */
typedef enum { RATEL_STAGING_PIPELINED = 0, RATEL_STAGING_SERIALIZED = 1, RATEL_STAGING_ZERO_COPY = 2 } ratel_staging;

/* Collectives: AUTO = NCCL when world_size > 1; NCCL = also for world_size 1
 * (a one-rank communicator: exercises the NCCL calls on one GPU); NONE = no
 * collectives at all -- each rank updates only its slices and the caller
 * moves the P16 slices itself (simulation/testing of the partition without
 * NCCL; clipping then uses the rank-local norm). */
typedef enum { RATEL_COMM_AUTO = 0, RATEL_COMM_NONE = 1, RATEL_COMM_NCCL = 2 } ratel_comm;

/* Update-kernel variants (same per-element arithmetic, bitwise-identical results):
 * TMA      bulk-copy (TMA) shared-memory pipeline, one 224 KB CTA per SM, the fastest alone (ranges with
 *          peer grads, ratel_register_peer_grads: the TMA-staged fused-reduction kernel);
 * LDG      register-staged 128/256-bit loads, 2 CTAs per SM, no shared memory (also selects the
 *          register-staged fused-reduction kernel);
 * LDG_LITE register-staged, one octet in flight per thread, <= 64 registers, 4 CTAs per SM, no shared
 *          memory: small enough to share an SM with a backward GEMM CTA while AGO overlaps them. */
typedef enum { RATEL_UPDATE_TMA = 0, RATEL_UPDATE_LDG = 1, RATEL_UPDATE_LDG_LITE = 2 } ratel_k1_kernel;

/* SSD tier I/O schedule.  DUPLEX: the reader (file -> staging) and the writer
 * (staging -> file) threads run freely, the device's queue mixes reads and
 * writes.  SIMPLEX: the paper's schedule for a simplex SSD link (Fig. 3b,
 * P:L1128-1131): one transfer at a time, and the write-back of
 * tile k starts only after the read of tile k+1 (or once no read is pending),
 * i.e. R0 R1 W0 R2 W1 R3 W2 ... -- "Main->SSD of tensor i after SSD->Main of
 * tensor i-1", at tile granularity. */
typedef enum { RATEL_SSD_DUPLEX = 0, RATEL_SSD_SIMPLEX = 1 } ratel_ssd_schedule;

/* SSD tier I/O method.  PREAD: each thread moves a tile's three arrays with
 * blocking pread/pwrite, one request at a time.  URING: each thread owns an
 * io_uring (raw syscalls) and keeps up to 32 requests of <= 4 MiB in flight
 * (queue depth > 1, what an NVMe needs to reach its bandwidth); a kernel that
 * refuses io_uring makes the first SSD registration fail with RATEL_EIO. */
typedef enum { RATEL_SSD_IO_PREAD = 0, RATEL_SSD_IO_URING = 1 } ratel_ssd_io;

typedef struct {
  int mode;               /* ratel_mode; default RATEL_ADAMW */
  double max_grad_norm;   /* > 0 enables the global L2-norm clip (torch clip_grad_norm_); default 0 */
  int pipeline_depth;     /* pinned-host tile ring depth (slots of {theta,m,v} tiles), 2..16; default 4 */
  int staging;            /* ratel_staging; default PIPELINED */
  uint64_t tile_elems;    /* pinned-host tile length in elements, multiple of 8; default 1<<24 */
  int max_ctas;           /* cap on the update kernel's grid (0 = SMs x resident CTAs) */
  int timing;             /* 1: bracket every update-kernel launch with CUDA events (ratel_kernel_timing) */
  int comm;               /* ratel_comm; default RATEL_COMM_AUTO */
  int host_threads;       /* HOST_COMPUTE handler threads (0 = OpenMP default: all cores) */
  int update_streams;     /* device-residency updates alternate over this many low-priority streams,
                             1..2; default 2: block b+1's update starts on the SMs block b's tail
                             frees instead of after it (results are identical) */
  int cta_tiles;          /* update-kernel tiles (4096 elements) per CTA.  0 (default): a persistent
                             grid (one CTA per SM, max_ctas cap) taking tiles dynamically -- fastest
                             alone.  > 0: a non-persistent grid of ceil(tiles / cta_tiles) CTAs, each
                             retiring after its cta_tiles tiles, so kernels of higher-priority streams
                             (the caller's backward) take SMs back within microseconds instead of
                             waiting for a persistent CTA; max_ctas is ignored.  Results are identical. */
  int k1_kernel;          /* ratel_k1_kernel: which update kernel (device-resident and tile updates);
                             default RATEL_UPDATE_TMA.  Results are identical. */
  int ssd_schedule;       /* ratel_ssd_schedule: RATEL_SSD* tiers; default RATEL_SSD_DUPLEX.  Results are
                             identical. */
  int ssd_io;             /* ratel_ssd_io: how the SSD tier's threads move tiles; default RATEL_SSD_IO_PREAD.
                             Results are identical. */
} ratel_config;

/* One contiguous parameter range of a block (a flat tensor, or a block's
 * whole flat parameter buffer).  Element i of the range is (param[i],
 * grad[i], master/exp_avg/exp_avg_sq[i - slice_begin]).
 *   param_bf16   device; the FULL range, capacity ratel_padded_numel(numel, N)
 *                elements (pads zero); this rank writes its slice and, when
 *                N > 1, the bf16 all-gather fills the rest in place.
 *   grad_bf16    device; the full range, or only this rank's slice when
 *                grad_is_rank_slice = 1 (e.g. a reduce-scatter output).
 *   master, exp_avg, exp_avg_sq
 *                fp32, THIS RANK'S SLICE ONLY (ratel_rank_slice), on the
 *                device (RATEL_DEVICE) or in page-locked host memory
 *                (RATEL_PINNED_HOST; cudaHostAlloc'd or cudaHostRegister'ed).
 *   numel        true length of the range (> 0).
 *   apply_weight_decay  0 exempts the range from weight decay (biases, LN).
 * All five pointers must be 16-byte aligned. */
typedef struct {
  void* param_bf16;
  const void* grad_bf16;
  int grad_is_rank_slice;
  float* master;
  float* exp_avg;
  float* exp_avg_sq;
  uint64_t numel;
  int apply_weight_decay;
} ratel_range;

/* Fills *cfg with the defaults listed above. */
void ratel_default_config(ratel_config* cfg);

/* Writes a 128-byte NCCL unique id (rank 0 calls it and broadcasts the bytes
 * through the caller's process group).  RATEL_ENCCL if NCCL cannot be loaded.
 * (Multi-GPU bootstrap: the paper's multi-GPU setting, §V-G, uses
 * no particular mechanism; NCCL over NVLink per BASELINE.json's north star.) */
int ratel_get_nccl_unique_id(void* out128);

/* Fig. 4's `Ratel_init()` (§IV-E): creates the
 * optimizer/copy/comm streams (the optimizer stream at the
 * lowest priority), events and, for world_size > 1, the NCCL communicator.
 * device: CUDA ordinal this process drives.  nccl_unique_id: 128 bytes, NULL
 * when world_size == 1 (or cfg->comm == RATEL_COMM_NONE).  cfg: NULL = defaults.  RATEL_ESTATE if already
 * initialised; RATEL_ECUDA if no usable device. */
int ratel_init(int device, int rank, int world_size, const void* nccl_unique_id,
               const ratel_config* cfg);

/* Fig. 4's `Ratel_Optimizer(...)` wrapping: registers the model
 * states of one handler unit -- the paper's "tensor i" / transformer block
 * (P:L1038-1041), P32 + OS32 + G16 + P16 of Table II.
 * Registers block `block_id` (0 <= id < RATEL_MAX_BLOCKS, each id once) made
 * of n_ranges (1..RATEL_MAX_RANGES_PER_BLOCK) ranges, all with the given
 * residency (ratel_residency).  Validates pointer kinds (device pointers on
 * this device; pinned host for RATEL_PINNED_HOST / RATEL_HOST_COMPUTE --
 * pageable memory is RATEL_EINVAL), alignment and sizes.  HOST_COMPUTE blocks
 * get library-owned pinned G16/P16 staging (4 B/param of the rank slice).  The ranges array is copied.  Not
 * allowed while a step is in flight (RATEL_ESTATE). */
int ratel_register_block(int block_id, const ratel_range* ranges, int n_ranges, int residency);

/* Fused update + all-gather over peer memory (multi-GPU).  peer_params[q]
 * (q = 0..world_size-1) is rank q's param_bf16 buffer of range `range_idx`
 * of block `block_id`, as mapped into THIS process (CUDA IPC, P2P or
 * torch.distributed._symmetric_memory buffer pointers); entry [rank] and
 * NULL entries are skipped.  From then on the update kernel stores this
 * rank's P16 slice of that range directly into every peer's buffer (NVLink
 * P2P stores inside the kernel, overlapping the HBM streaming) and the NCCL
 * all-gather of that range is skipped.  Synchronisation (NCCL communicator
 * present): each hand-off of such a block adds an 8-byte allreduce on the
 * comm stream and the block's update waits for it -- every rank has handed
 * the block off, so no rank's backward still reads the P16 the peers are
 * about to overwrite -- and ratel_sync adds one more as the "all peer stores
 * landed" barrier.  With RATEL_COMM_NONE the caller provides that ordering.
 * Not for RATEL_HOST_COMPUTE blocks.  Between steps only.  The pointers are
 * borrowed like all registered memory. */
int ratel_register_peer_params(int block_id, int range_idx, void* const* peer_params, int n);

/* Fused data-parallel gradient reduction (reduce-scatter folded into the
 * update, reading R17 -- the paper leaves the
 * multi-GPU gradient semantics unspecified).  rank_grads[q]
 * (q = 0..world_size-1, world_size <= 8) is rank q's LOCAL full-range bf16
 * gradient of range `range_idx` of block `block_id` (numel elements, as mapped
 * into THIS process: CUDA IPC, P2P or symmetric-memory pointers; entry [rank]
 * is ignored -- the range's own grad_bf16 is used).  From then on the update
 * of this rank's slice uses
 *     g[i] = fp32( grad_scale * sum_{q=0..N-1} bf16(G16_q[i]) )
 * (fp64 sum in rank order, one rounding; grad_scale = 1/N is the DDP mean, 1
 * the sum), also for the clip norm.  The range must have grad_is_rank_slice
 * = 0; not for RATEL_HOST_COMPUTE blocks (RATEL_EINVAL); grad_scale finite >
 * 0.  Synchronisation (NCCL communicator present): each hand-off adds an
 * 8-byte allreduce on the comm stream before the block's update -- the
 * cross-rank "all G16 of this block are complete" barrier -- and ratel_sync's
 * barrier keeps every G16 unmodified until all ranks finished reading it;
 * ratel_block_wait on such a block is then collective (every rank calls it
 * for the same blocks in the same order).  With RATEL_COMM_NONE the caller
 * provides that ordering.  Between steps only; pointers are borrowed. */
int ratel_register_peer_grads(int block_id, int range_idx, const void* const* rank_grads, int n,
                              double grad_scale);

/* SSD residency (RATEL_SSD): attach the state file of range
 * `range_idx` of block `block_id`.  The rank slice's theta, m and v are fp32
 * arrays in the file at `offset`, `offset + S` and `offset + 2S`, with
 * S = ratel_ssd_range_bytes(numel, world, rank) / 3 (each array padded to a
 * multiple of 4096 bytes; the padding is read and written back unchanged).
 * fd: open for reading and writing (O_RDWR), borrowed until ratel_finalize;
 * open it with O_DIRECT to bypass the page cache (the measured numbers do);
 * offset: multiple of 4096; the file must already hold offset + 3S bytes and
 * the initial states (the caller writes theta0, m = v = 0).  Requires
 * cfg.tile_elems to be a multiple of 1024.  Every range of an SSD block
 * needs a file before its first hand-off (RATEL_ESTATE otherwise).  Between
 * steps only.  RATEL_EINVAL on a bad fd, alignment or short file.  With SSD
 * blocks, ratel_sync (either form) also waits on the host until every state
 * write-back of the step has reached the file. */
int ratel_register_ssd(int block_id, int range_idx, int fd, uint64_t offset);

/* Bytes one range's states take in an SSD state file (3 x 4096-padded fp32
 * arrays of the rank's slice; 0 for an empty slice).  Pure host function. */
uint64_t ratel_ssd_range_bytes(uint64_t numel, int world_size, int rank);

/* The optimizer of the iteration (Adam [44]; §II):
 * arms optimizer step `step` (1-based t, strictly increasing across steps)
 * with the given hyperparameters (0 <= beta < 1, lr, eps, wd >= 0, finite).
 * Blocks already handed off in this step are enqueued now (deferred mode);
 * blocks handed off later are enqueued at their hand-off (AGO). */
int ratel_adam_step(double lr, double beta1, double beta2, double eps, double weight_decay,
                    int64_t step);

/* Active gradient offloading's "active message" (§IV-C: the
 * handler of tensor i runs "upon ... receiving the offloaded gradients",
 * which arrive "with a decreasing index") for block `block_id`: its gradient is complete on
 * `stream` (a cudaStream_t, NULL = legacy default stream).  Records an event
 * on `stream`; the optimizer stream waits on it -- no host blocking, no data
 * movement.  RATEL_ESTATE if the block was already handed off this step or
 * is not registered. */
int ratel_offload_grad_chunk(int block_id, void* stream);

/* Orders `stream` (cudaStream_t) after the update of block `block_id` that
 * last consumed its gradient: once it returns, work on `stream` may overwrite
 * that block's grad buffer (and read its P16 slice).  This is what lets a
 * caller recycle a small ring of gradient buffers during backward -- the
 * memory side of active gradient offloading: a block's G16 is dead as soon as
 * its handler ran.  RATEL_ESTATE if the block was handed off
 * in the current step but its update is not enqueued yet (deferred mode) or
 * it is not registered.  RATEL_SSD blocks: the library's reader thread issues
 * the block's grad reads on its own streams, so until ratel_block_wait (which
 * waits on the host until the reader has issued them, then orders `stream` and
 * the optimizer stream after them) or ratel_sync, record_stream on the
 * optimizer stream does not cover them -- keep the grad alive until then. */
int ratel_block_wait(int block_id, void* stream);

/* Ends the step: `stream` (cudaStream_t) is ordered after every update,
 * write-back and all-gather of the step, so the next forward on it reads the
 * updated P16 (no staleness, footnote 4 P:L1147-1152).  stream == NULL
 * blocks the host instead.  RATEL_ESTATE if the step is armed but some
 * registered block was not handed off (or vice versa).  In clip mode a
 * blocking sync returns RATEL_ENONFINITE if the global norm was not finite. */
int ratel_sync(void* stream);

/* End of training (the exit of Fig. 4's `with Ratel_init():`):
 * waits for outstanding work, destroys everything the library created and
 * clears all registrations and the sticky error. */
int ratel_finalize(void);

/* Message describing the last error on this thread ("" if none). */
const char* ratel_last_error(void);

/* Range partition of the multi-GPU path (north star: "each GPU owning a
 * contiguous shard of optimizer state", R12).
 * Capacity of a range's param buffer for world_size ranks: numel rounded up
 * to a multiple of 8*world_size (each rank's slice is a multiple of 8
 * elements, keeping 16-byte alignment).  Pure host function. */
uint64_t ratel_padded_numel(uint64_t numel, int world_size);

/* This rank's slice [*begin, *end) of a range of numel elements:
 * s = ratel_padded_numel(numel, N)/N, begin = min(numel, rank*s),
 * end = min(numel, begin + s).  Pure host function. */
int ratel_rank_slice(uint64_t numel, int world_size, int rank, uint64_t* begin, uint64_t* end);

/* Rebuilds block `block_id`'s working copy from its master weights:
 * P16[slice] = bf16_rne(master) for this rank's slice of every range (the
 * same RNE conversion the update uses, "produces a 16-bit
 * parameter copy"), then -- N > 1 -- the bf16 all-gather (NCCL in place, or
 * the peer stores of ratel_register_peer_params plus an 8-byte barrier), so
 * every rank's full P16 matches the restored masters.  For checkpoint resume
 * (restore master/m/v, then call this for every block) or any out-of-band
 * change of the masters.  Ordered after the work already on `stream`
 * (cudaStream_t); `stream` is ordered after the refresh (NULL: the host
 * blocks until done).  Device, pinned-host and HOST_COMPUTE masters are read
 * in place; RATEL_SSD masters are read from the state file (the calling
 * thread preads tile by tile).  Between steps only (RATEL_ESTATE otherwise);
 * collective when world_size > 1 (every rank, same blocks, same order). */
int ratel_refresh_params(int block_id, void* stream);

/* The optimizer stream (cudaStream_t) -- for torch's record_stream. NULL before init. */
void* ratel_optimizer_stream(void);

/* Blocking: the global sum of squared gradients of the last clip-mode step
 * (after the allreduce; clipping per DESIGN.md R9 -- the paper is silent,
 * the north star asks for "optional grad-norm clipping").  RATEL_ESTATE if
 * clipping is off. */
int ratel_get_grad_sumsq(double* out);

/* Page-locked host memory for RATEL_PINNED_HOST / RATEL_HOST_COMPUTE states
 * (the paper keeps P32/OS32 off the GPU, §III-A):
 * exactly `bytes` (cudaHostAlloc, portable), 64-byte aligned; *out = NULL on
 * failure (RATEL_ENOMEM, not sticky).  Frameworks' pinned allocators may round
 * large blocks up (torch: powers of two), which does not fit 100+ GB of
 * states into host RAM; registering pageable memory instead measured ~10 %
 * slower on the host link.  Free with ratel_free_pinned.  Neither call needs
 * ratel_init. */
int ratel_alloc_pinned(uint64_t bytes, void** out);
int ratel_free_pinned(void* p);

/* Busy time of the update kernels (ms) -- the union of the event-timed
 * [start, end] intervals of every launch, so overlapping launches on the two
 * update streams are not double counted -- and the number of timed launches
 * since the last reset (requires cfg.timing = 1; blocking). */
int ratel_kernel_timing(double* total_ms, int64_t* launches, int reset);

/* Number of kernels this library launched since init (update, grad-norm
 * partial and finalize kernels). */
int64_t ratel_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* RATEL_H */
