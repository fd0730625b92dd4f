/*
 * sh.h -- C ABI of the STRONGHOLD working-window offload engine (B200 / sm_100a).
 *
 * The engine trains a layer-sequential model whose parameters, gradients and Adam
 * states live in pinned host RAM while only a sliding window of layers sits in a
 * ring of GPU layer slots (§III-A; §III-C,
 * Fig. 3b/3c).  The caller's model code drives it through per-layer hooks, the way
 * STRONGHOLD's pre_forward / post_forward / pre_backward callbacks are driven by
 * framework hooks.
 *
 * Step protocol (any other order returns SH_ERR_STATE):
 *     for i in 0..L-1:    sh_forward_layer(i, SH_PRE)  -> compute FP of layer i -> sh_forward_layer(i, SH_POST)
 *     (caller: head / loss using sh_resident views)
 *     for i in L-1..0:    sh_backward_layer(i, SH_PRE) -> recompute + BP of layer i -> sh_backward_layer(i, SH_POST)
 *     (caller: embedding backward into the sh_resident grad views)
 *     sh_step()
 * Every device pointer handed out is valid on the caller's compute stream between
 * the PRE that returned it and the matching POST (layers) or the next sh_step
 * (resident set).  The caller must enqueue its layer computation on that compute
 * stream.  Hooks never block the host on the GPU; they may block on a true data
 * dependency (the CPU Adam update of a layer that is about to be prefetched, or a
 * full host landing ring).
 *
 * Window convention (eq. 1b-1c are garbled; reading R4):
 *   window w = the paper's m = prefetch distance.  The ring has w+1 slots (the
 *   extra slot is the landing slot s^j of (1c)).  Layers [0, w) plus the resident
 *   set (embedding, positions, final LN) are GPU-optimised ("the first few layers
 *   ... layers of the first working window"; Fig. 3 caption
 *   PAPER.md:130).  Layers [w, L) are host-optimised by the multi-threaded CPU AdamW
 *   (PAPER.md:201-205).  w = L is the all-resident configuration; w = 0 is
 *   serial fetch-then-compute (L2L-like).
 *
 * Numerics contract (makes results bit-identical for
 * every window): the GPU Adam (K2) and the CPU Adam execute per
 * element, in IEEE fp32 round-to-nearest, no FTZ/DAZ:
 *     g = g*coef (only when clipping is on);  m = fma(b1, m, omb1*g);
 *     v = fma(b2, v, omb2*(g*g));  d = sqrt(v)/sqrt_bc2 + eps;
 *     p = fma(-step_size, m/d, wd ? p*decay : p);  p16 = rna_bf16(p)
 *   with b1, b2, eps, omb1 = 1-b1, omb2 = 1-b2, sqrt_bc2 = sqrt(1-b2^t), step_size = lr/(1-b1^t),
 *   decay = 1 - lr*lambda computed in double from the double hyperparameters on the host and
 *   rounded once to fp32.
 *   rna_bf16 is round-to-nearest, ties away from zero: (bits(p) + 0x8000) >> 16, canonical NaN 0x7FC0
 *   (R25: the rounding under which the split master below is lossless).
 *
 * bf16 host layout (default, R25): a host-optimised layer keeps its fp32 master as two 16-bit
 *   planes, hi = rna_bf16(p) -- which IS the compute copy the prefetch moves, 2 B/param -- and lo = the
 *   low 16 bits of bits(p); p = (hi << 16) + sext16(lo) exactly (a NaN comes back as a NaN).  12 B/param of
 *   host RAM (hi, lo, m, v) with a 2 B/param fetch and no shadow copy.  SH_FLAG_FETCH_FP32 keeps an fp32
 *   master (fetch 4 B + K1 cast on the GPU), SH_FLAG_BF16_SHADOW an fp32 master + a bf16 shadow (14 B).
 *
 * Errors: every call returns sh_status; no exception crosses the ABI.  The message
 * of the last failing call on this thread is sh_last_error().  After SH_ERR_CUDA /
 * SH_ERR_NCCL / SH_ERR_OOM_* inside a step, the context is failed: every call except
 * sh_destroy, sh_stats and sh_last_error returns SH_ERR_STATE.
 * Threading: one driver thread per context.  Internally the engine runs an H2D
 * issuer thread, a D2H issuer thread and the CPU Adam pool.
 */
#ifndef SH_H_
#define SH_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SH_ABI_VERSION 3  /* 2: sh_stats_t / sh_profile grew (round 2), bf16 rounding RNA, split host master;
                            3: sh_config.hybrid_layers, sh_stats_t hybrid counters, sh_op_adamw_split_gpu */

typedef struct sh_ctx sh_ctx;

typedef enum {
  SH_OK = 0,
  SH_ERR_INVALID = -1,     /* bad argument / configuration (message says which) */
  SH_ERR_CUDA = -2,        /* CUDA runtime error (sync or async) */
  SH_ERR_OOM_DEVICE = -3,  /* device allocation failed */
  SH_ERR_OOM_HOST = -4,    /* host allocation or page-locking failed */
  SH_ERR_NCCL = -5,        /* NCCL error (world_size > 1) */
  SH_ERR_STATE = -6,       /* call out of protocol order, or context failed */
  SH_ERR_UNSUPPORTED = -7  /* feature not available on this build / device */
} sh_status;

typedef enum { SH_FP32 = 0, SH_BF16_MIXED = 1 } sh_precision;
typedef enum { SH_PRE = 0, SH_POST = 1 } sh_phase;

/* What sh_read_layer returns. */
typedef enum {
  SH_READ_PARAM = 0,   /* fp32 master parameters (float[numel]) */
  SH_READ_M = 1,       /* fp32 Adam first moment */
  SH_READ_V = 2,       /* fp32 Adam second moment */
  SH_READ_COMPUTE = 3, /* compute copy: uint16 bf16 bits (bf16 mode) or float (fp32 mode) */
  SH_READ_GRAD = 4     /* fp32 gradients of the last step (host layers: from the landing buffer,
                          SH_ERR_STATE if the ring has reused it) -- diagnostics / parity tests */
} sh_read_what;

/* One layer (offload unit): its tensors in the caller's order.
 * numel[k] > 0.  weight_decay[k] != 0: decoupled decay applies to tensor k. */
typedef struct {
  int32_t n_tensors;             /* 1..64 */
  const int64_t* numel;          /* [n_tensors] */
  const uint8_t* weight_decay;   /* [n_tensors] */
} sh_layer_shape;

/* Flags */
#define SH_FLAG_PROFILE   (1ull << 0) /* record per-layer CUDA events every step (else warm-up only) */
#define SH_FLAG_POISON    (1ull << 1) /* debug: fill a slot's param half with NaN before every refill */
#define SH_FLAG_DUPLEX    (1ull << 2) /* autotuner: full-duplex link, max() instead of sum in (1d)/(2d) */
#define SH_FLAG_FETCH_FP32 (1ull << 5) /* bf16 mode: no host bf16 shadow (12 instead of 14 B/param of host
                                          RAM); prefetch the fp32 master (4 B/param over the link) into
                                          the slot's idle grad half and K1-cast it on the GPU */
#define SH_FLAG_TEST_NO_COLLECTIVE (1ull << 6) /* test: world_size > 1 without NCCL (all ranks feed identical
                                                  data, so the average is the local gradient); exercises
                                                  the shared store / slicing with several processes */
#define SH_FLAG_SLICE_FETCH (1ull << 7) /* NEXT-1 (data parallel + shm_name): each rank H2Ds only its 1/W
                                           slice of a fetched layer; an in-place ncclAllGather over NVLink
                                           assembles the layer in every rank's slot (PCIe bytes and host
                                           DRAM reads per rank / W).  Needs NCCL >= 2.18 (ncclCommSplit). */
#define SH_FLAG_DELAY_INJECT (1ull << 8) /* test: random 0-2 ms sleeps in the copy issuers and CPU Adam tasks
                                            (ordering-race hunting; results must stay bitwise identical) */
#define SH_FLAG_DECOUPLE  (1ull << 9) /* autotuner: decouple the ring (prefetch distance) from the
                                         GPU-optimised set (needs no clipping and a landing buffer per
                                         layer, grad_ring_depth 0; R22) */
#define SH_FLAG_SPILL_EVICT (1ull << 10) /* NEXT-2, no effect since ABI round 2: the spill tier always reads and
                                           writes its files with O_DIRECT (no page cache), so the RAM it holds
                                           is bounded by its pinned staging buffers */
#define SH_FLAG_TEST_DP_PATH (1ull << 11) /* test: take the data-parallel path at world_size 1 (one-rank NCCL
                                            communicator from nccl_unique_id: the per-layer and resident
                                            all-reduces run on the comm stream and are the identity) */
#define SH_FLAG_KEEP_GRADS (1ull << 12) /* diagnostics: one gradient buffer per GPU-optimised layer (no clipping),
                                          so SH_READ_GRAD can return every layer's gradients after a step
                                          (default: a rotation of 2, or 4 with data parallelism) */
#define SH_FLAG_ABLATE_ALLOC (1ull << 13) /* ablation (Fig. 14): a cudaMalloc/cudaFree pair per
                                            prefetch, as per-layer CUDA-allocator buffers would cost */
#define SH_FLAG_GROW_LANDING (1ull << 14) /* autotuner (private store, grad_ring_depth < n_layers): after the
                                            window is applied, grow the landing ring to one buffer per
                                            host-optimised layer in the host RAM the layers joining the GPU
                                            set gave back (no D2H waits on the CPU Adam), and allow the
                                            decoupled ring (R22, with SH_FLAG_DECOUPLE), which needs it */
#define SH_FLAG_FILL_GPU (1ull << 15)     /* autotuner, decoupled: the GPU-optimised set takes all the HBM the ring
                                            leaves (sh_profile.fill_gpu) */
#define SH_FLAG_LATE_SHADOW (1ull << 16)  /* bf16 mode with SH_FLAG_FETCH_FP32: after the autotune, give every host
                                            layer a bf16 shadow in the host RAM the GPU set gave back (fetch 2
                                            instead of 4 B/param; the solver already plans with that cost) */
#define SH_FLAG_TEST_HOST_COLLECTIVE (1ull << 17) /* test (data parallel with shm_name): every collective -- the
                                            per-layer all-reduce / reduce-scatter, the resident all-reduce,
                                            the norm-partials all-gather -- runs through a shared host segment
                                            on the driver thread, the ranks' contributions summed in rank
                                            order (identical on every rank).  Several ranks on ONE GPU with
                                            DIFFERENT data: the averaging itself is checked against the
                                            oracle's global-batch mean.  No NCCL. */
#define SH_FLAG_BF16_SHADOW (1ull << 18) /* bf16 mode: fp32 master + separate bf16 shadow in host RAM (14 B/param)
                                           instead of the split master (the round-1 layout) */
#define SH_FLAG_CPU_HARD  (1ull << 4) /* autotuner: CPU-update throughput (eq. 3, R19) is a hard constraint */
#define SH_FLAG_SYNC_CPU  (1ull << 3) /* debug: run each CPU Adam task inline when its grads land (no pool; ignored in clip mode) */

typedef struct {
  int32_t n_layers;                 /* L >= 1, execution order */
  const sh_layer_shape* layers;     /* [n_layers] */
  sh_layer_shape resident;          /* embedding / positions / final LN: always in HBM */
  int32_t window;                   /* 0..n_layers, or -1: w0 = min(2, w_max) then autotune after warm-up */
  int32_t precision;                /* sh_precision */
  double lr;                        /* initial learning rate (sh_set_lr changes it) */
  double beta1, beta2, eps, weight_decay;  /* doubles: the per-step scalars are derived in double */
  double max_grad_norm;             /* <= 0: no clipping (throughput mode, R3) */
  int32_t device;                   /* CUDA ordinal */
  void* compute_stream;             /* caller-owned cudaStream_t for all layer compute (required) */
  int32_t cpu_threads;              /* CPU Adam threads; 0 = all online cores */
  int32_t grad_ring_depth;          /* host landing buffers for offloaded grads; 0 = one per host layer */
  int32_t warmup_steps;             /* profiled steps before autotune (default 5); 0 = default */
  int64_t device_budget_bytes;      /* S_avail for ring + G states; 0 = free memory - 2 GiB */
  double cpu_util_max;              /* autotuner eq. 3 utilisation target rho (SH_FLAG_CPU_HARD); 0 = 0.85 */
  int32_t ring_slots;               /* ring size cap (0: window + 1).  Without clipping a GPU-optimised
                                       layer is updated right after its backward, so its slot is not
                                       pinned and the ring may be smaller than the GPU-optimised set:
                                       prefetch distance = min(window, ring_slots - 1) (R22) */
  int32_t world_size;               /* data-parallel ranks (1 = single GPU) */
  int32_t rank;
  const void* nccl_unique_id;       /* 128-byte ncclUniqueId, required when world_size > 1 */
  uint64_t flags;                   /* SH_FLAG_* */
  const char* shm_name;             /* world_size > 1: name of ONE shared host store for all ranks of the
                                       box (/dev/shm); rank r offloads and CPU-updates only
                                       slice r of every layer.  NULL/"": a private replica per rank */
  int32_t n_executors;              /* NEXT-3 multi-stream executors (Fig. 5): K >= 2
                                       concurrent training workers on one GPU share ONE copy of every
                                       layer's parameters (the ring slot) and each computes a micro-batch
                                       on its own stream; executor e >= 1 writes its gradients into the
                                       engine-owned buffers of sh_executor_grads, and the engine's K4
                                       kernel averages them into executor 0's buffers ("an all-reduce
                                       operation to synchronize the gradients among parallel training
                                       workers before performing parameter updates") at
                                       the backward POST (layers) and at sh_step (resident set).
                                       0 or 1: a single worker.  At most 8. */
  const char* spill_dir;            /* NEXT-2 secondary-storage tier: NULL/"" = off.
                                       Otherwise a directory (NVMe or any file system): host-optimised
                                       layers whose pinned block would exceed host_pin_budget_bytes, or
                                       for which pinned host RAM runs out, are kept in files there,
                                       memory-mapped (MAP_SHARED) instead of pinned ("memory-mapping a
                                       swap file on the secondary storage to the CPU memory space").
                                       Files are read and written with O_DIRECT bulk requests through
                                       io_uring ("asynchronous bulk read/write requests"),
                                       no page cache: a prefetch reads the layer's fetch region into one
                                       of two pinned bounce buffers, then H2D; when its gradients land
                                       a spill-read thread reads master / m / v into one of
                                       SH_SPILL_STAGING (env, default 3) pinned staging copies, the CPU
                                       Adam updates that copy, a spill-write thread writes master / m /
                                       v / shadow back, and only then is the layer updated for the next
                                       fetch.  Results are bit-identical to the all-pinned store.  Files
                                       are created O_EXCL, unlinked at once, space reserved with
                                       posix_fallocate; file systems without O_DIRECT get the same
                                       aligned transfers through the page cache.  Not with shm_name. */
  int64_t host_pin_budget_bytes;    /* cap on pinned host-store bytes (layer blocks + landing ring);
                                       0 = no cap (spill only when pinning fails for lack of RAM) */
  int32_t warmup_window;            /* window of the warm-up steps when window == -1 (0: min(2, n_layers)).
                                       Only host-optimised layers hold a host block (a layer joining the
                                       GPU set gives its block back), so a larger warm-up window lowers
                                       the host RAM the store needs from the start */
  int32_t numa_policy;              /* SH_NUMA_*: where the pinned host store lives and which cores update
                                       it.  0 = SH_NUMA_AUTO */
  int64_t ring_bytes;               /* NEXT-4 fixed-byte window: 0 = off (w + 1 slots sized for
                                       the largest layer).  > 0: ONE device buffer of at most ring_bytes
                                       holding variable-capacity slots -- slot 0 fits the largest layer,
                                       slot x >= 1 is sized for layer x (execution order) while the bytes
                                       last -- and the prefetch runs ahead until no evictable slot fits
                                       the next layer, so the number of buffered layers follows the
                                       layer sizes (heterogeneous stacks).  window still sets the
                                       GPU-optimised set.  Needs no clipping, world_size 1, window >= 0,
                                       ring_slots 0; SH_ERR_INVALID if the largest layer does not fit */
  int32_t hybrid_layers;            /* R28 hybrid update: the lowest `hybrid_layers` host-optimised layers
                                       (w .. w+hybrid_layers-1) keep their states in host RAM but are
                                       updated on the GPU: their lo / m / v planes are fetched into HBM
                                       staging during the backward, K2S updates the split master right
                                       after the layer's backward (the compute copy in its ring slot in
                                       place), and hi / lo / m / v are written back to host RAM; the updated
                                       compute copy stays in the ring for the next forward.  Takes the CPU
                                       AdamW of the layers the next forward needs first off the step
                                       boundary (eq. 3).  Bitwise the CPU update.  Needs
                                       the split host master (bf16 mode), no clipping, world_size 1, no
                                       spill tier, no fixed-byte ring; 0 = off */
} sh_config;

/* NUMA placement policies (sh_config.numa_policy).  Placement is an mbind(2) before the first
 * touch (MPOL_PREFERRED: a full node spills to another instead of failing); CPU Adam workers are
 * pinned with pthread_setaffinity_np.  On a single-node host every policy is a no-op. */
#define SH_NUMA_AUTO 0        /* SPLIT for a private store on a multi-node host; LOCAL with data
                                 parallelism (shared store: slice r on GPU r's node) */
#define SH_NUMA_SPLIT 1       /* layer x's block on node x mod n_nodes; workers spread over the nodes in
                                 proportion to their cores, each preferring the jobs of its own node's
                                 layers (takes others only when it would idle); landing buffers
                                 interleaved */
#define SH_NUMA_LOCAL 2       /* every block on the GPU's node (PCI numa_node of the device), workers
                                 pinned to that node (cpu_threads 0 = that node's cores) */
#define SH_NUMA_INTERLEAVE 3  /* every block page-interleaved over all nodes, workers unpinned */
#define SH_NUMA_NONE 4        /* first touch only */

/* Per-layer profile consumed by the window solver (PAPER.md:132 notation; times in ms,
 * sizes in bytes).  Arrays have n_layers entries; NULL arrays are treated as zeros. */
typedef struct {
  int32_t n_layers;
  const double* t_fp;       /* FP compute time of layer i */
  const double* t_bp;       /* BP time incl. recompute (PAPER.md:153 fn. 2) */
  const double* t_c2g;      /* host -> device fetch of layer i */
  const double* t_g2c;      /* device -> host gradient offload of layer i */
  const double* t_stage;    /* K1 restage of a GPU-optimised layer in BP (replaces t_c2g for i < w) */
  const double* t_opt_gpu;  /* K2 time of layer i */
  const double* t_opt_cpu;  /* CPU Adam time of layer i */
  double t_async;           /* one asynchronous hook call (eq. 4) */
  const int64_t* slot_bytes;   /* s_bp of layer i: bytes of one ring slot holding i (param + grad half) */
  const int64_t* gstate_bytes; /* HBM bytes of layer i's master/m/v when GPU-optimised */
  int64_t fixed_bytes;         /* HBM always used by the engine (resident set, scratch) */
  int64_t s_avail;             /* S_avail */
  int32_t duplex;              /* 1: soft constraints use max(Σc2g, Σg2c) (R7) */
  int32_t cpu_hard;            /* 1: also require the CPU-update throughput form of eq. 3 (R19):
                                  Σ_{k>=w} t_opt_cpu^k <= rho * (Σ_i (t_fp^i + t_bp^i) + Σ_{i<w} t_opt_gpu^i) */
  double cpu_util_max;         /* rho in (0, 1]; <= 0 means 1 (utilisation target of the CPU pool) */
  int32_t decouple;            /* 1: choose the prefetch distance d (ring d+1, by P1/P2) and the
                                  GPU-optimised set g >= d (by eq. 3 + memory) separately (R22) */
  int32_t fp_serial;           /* 1: (1b) also in its serialised-link form (R23): the FP fetches of the host
                                  layers queue on one link, F(j) = max(F(j-1), S(j-d)) + t_c2g[j] <= S(j)
                                  with S(p) = Σ_{i<p} t_fp -- a hard constraint */
  int32_t fill_gpu;            /* decouple: g = the largest GPU-optimised set the memory leaves next to the
                                  ring (instead of the smallest meeting eq. 3) */
  int32_t landing_buffers;     /* host landing buffers (0: unknown).  With fill_gpu, when no ring meets the
                                  hard constraints (a link-bound FP, R27): the smallest ring whose gradient
                                  pool holds the BP backlog ceil(Σ_{k>=g} max(0, 1 - t_bp/t_opt_cpu)) -
                                  landing_buffers, the GPU set filling the rest (reason 3) */
} sh_profile;

typedef struct {
  int32_t window;          /* chosen w* */
  int32_t w_max_memory;    /* largest w meeting (1c)/(2c) */
  int32_t reason;          /* 0: hard+soft met (w < L); 1: hard only; 2: memory fallback;
                              3: link-bound FP, pool-sized decoupled ring + filled GPU set (R27) */
  int32_t fp_hard_ok, bp_hard_ok, soft_ok;  /* at the chosen window */
  double eq3_min_slack_ms; /* min_k [Σ_{i<=k}(t_fp+t_bp) + Σ_{i<w} t_opt_gpu - t_opt_cpu_k]  (eq. 3) */
  int32_t eq3_ok;
  double eq4_lhs_ms, eq4_rhs_ms; /* 5 n t_async  vs  Σ_{i=w}^{n-1} t_opt_gpu (eq. 4) */
  double cpu_total_ms;     /* Σ_{k>=w} t_opt_cpu^k at the chosen window */
  double gpu_step_ms;      /* Σ_i (t_fp^i + t_bp^i) + Σ_{i<w} t_opt_gpu^i */
  int32_t ring_slots;      /* chosen ring size (prefetch distance + 1); window + 1 unless decoupled */
} sh_solve_report;

typedef struct {
  int64_t step;                 /* completed sh_step calls */
  int32_t window;
  int32_t n_slots;
  int64_t host_bytes;           /* pinned host store */
  int64_t device_bytes;         /* ring + G states + resident + scratch */
  int64_t h2d_bytes, d2h_bytes; /* cumulative algorithmic bytes moved by the engine */
  int64_t h2d_copies, d2h_copies, stage_launches;
  double h2d_busy_ms, d2h_busy_ms; /* cumulative copy durations (profiled steps only) */
  int64_t h2d_profiled_bytes, d2h_profiled_bytes;
  double cpu_adam_ms;           /* cumulative wall time of CPU Adam tasks (summed over threads) */
  int64_t cpu_adam_elems;
  double cpu_wait_ms;           /* cumulative time the H2D issuer waited on CPU Adam (eq. 3 violation) */
  double k2_ms_last;            /* duration of the last sh_step K2 launch(es) when profiled */
  int64_t k2_bytes_last;        /* algorithmic HBM bytes of that K2 */
  int32_t k2_launches_last;
  int32_t cpu_threads;
  int32_t profiled_steps;
  double k2_ms_sum;             /* K2 durations summed over all profiled steps */
  int64_t k2_bytes_sum;         /* their algorithmic HBM bytes */
  int64_t k2_samples;           /* number of profiled K2 phases summed */
  double k3_ms_sum;             /* per-layer K3 (Σg²) durations summed (profiled steps) */
  int64_t k3_bytes_sum;
  int64_t k3_samples;
  /* copy/compute overlap of the last harvested profiled step (Fig. 4 analogue):
     |copy ∩ compute| / |copy| with compute = union of the per-layer FP/BP compute intervals */
  double h2d_overlap_frac, d2h_overlap_frac;
  double last_step_ms;          /* first FP hook .. end of K2 of that step (GPU time) */
  int64_t spill_bytes;          /* NEXT-2: bytes of host-optimised layer state in spill files */
  int32_t spilled_layers;       /* number of layers in the spill tier */
  int32_t landing_buffers;      /* host landing buffers for offloaded gradients (grows when the autotuner
                                   decouples the ring on a private store) */
  int32_t numa_nodes;           /* NUMA nodes of the host (sysfs) */
  int32_t numa_policy;          /* policy in effect (SH_NUMA_AUTO resolved) */
  int32_t numa_gpu_node;        /* node index of this context's GPU */
  int32_t numa_pinned_workers;  /* CPU Adam workers pinned to a node */
  int64_t numa_bound_bytes;     /* host-store bytes placed with mbind */
  double compute_busy_ms;       /* last harvested profiled step: union of the compute-stream intervals
                                   (layer FP/BP compute, K2); last_step_ms - compute_busy_ms is the
                                   compute stream's stall (waiting on fetches, restages, updates) */
  int64_t ring_bytes;           /* device bytes of the slot ring */
  int64_t cpu_adam_shadow_elems;  /* of cpu_adam_elems, those that also wrote a bf16 shadow (30 instead of
                                     28 B of host DRAM per element) */
  int32_t shadow_layers;        /* host-optimised layers holding a bf16 shadow (fetched at 2 B/param) */
  int32_t spill_direct;         /* NEXT-2: the spill files are O_DIRECT (0: the file system refused it) */
  int64_t spill_read_bytes;     /* NEXT-2: cumulative bytes read from / written to the spill files */
  int64_t spill_write_bytes;
  double spill_io_ms;           /* cumulative duration of those transfers (summed over the I/O threads) */
  int32_t spill_uring;          /* 1: transfers go through io_uring (else pread / pwrite) */
  int32_t hybrid_layers;        /* host layers updated on the GPU (sh_config.hybrid_layers, R28) */
  int64_t hybrid_updates;       /* cumulative K2S launches of the hybrid update */
  int64_t hybrid_h2d_bytes;     /* of h2d_bytes / d2h_bytes: the hybrid update's lo / m / v fetches and */
  int64_t hybrid_d2h_bytes;     /* hi / lo / m / v write-backs */
} sh_stats_t;

/* One interval of a profiled step (times in ms from the step's first FP hook). */
typedef struct {
  int32_t kind;   /* 0 FP compute, 1 BP compute, 2 H2D (FP), 3 H2D (BP), 4 D2H grads, 5 K1 stage,
                     6 K3 sumsq, 7 K2; host-clock intervals aligned to the step start: 8 CPU Adam job of
                     the layer (this step's gradients; runs into the next step), 9 H2D issuer waiting
                     for the CPU Adam of the layer it is about to fetch */
  int32_t layer;  /* -1 for K2 */
  double start_ms, end_ms;
} sh_trace_event;

/* ---- lifecycle ------------------------------------------------------------------ */

/* Validate cfg, build the size table (a0), allocate and page-lock the
 * host store (D1), reserve the ring of w+1 slots and the GPU states
 * once (D2), start the issuer threads and the CPU Adam pool.
 * Returns SH_ERR_INVALID for bad shapes, SH_ERR_OOM_* when memory is short. */
sh_status sh_init(const sh_config* cfg, sh_ctx** out);

/* Copy in the initial fp32 state of `layer` (-1 = resident set).  params / m / v are
 * host arrays of Σ numel floats, tensors concatenated in the caller's order; m and v
 * may be NULL (zeros).  `step` = number of updates already applied (0 for fresh
 * training; used for bias correction on resume).  Caller keeps ownership.  Must be
 * called for every layer and the resident set before the first forward hook. */
sh_status sh_register_host_store(sh_ctx* ctx, int32_t layer, const float* params,
                                 const float* m, const float* v, int64_t step);

/* Block until the engine is idle (all streams, issuers and CPU Adam tasks). */
sh_status sh_synchronize(sh_ctx* ctx);

sh_status sh_destroy(sh_ctx* ctx);

/* ---- hooks (hot path) ----------------------------------------------------------- */

/* FP hook.  SH_PRE: issue the async prefetch of the layer that enters the window
 * (PAPER.md:108 step 1; position c+w of the step's use sequence), make the compute
 * stream wait for layer `layer`'s arrival, and write its n_tensors device pointers
 * (bf16 in SH_BF16_MIXED, fp32 in SH_FP32) into dev_params.  SH_POST: mark the
 * layer's slot reusable once the compute enqueued so far finishes (step 3; no
 * parameter write-back: FP does not change parameters, R10). */
sh_status sh_forward_layer(sh_ctx* ctx, int32_t layer, int32_t phase, void** dev_params);

/* BP hook.  SH_PRE: as FP, plus a zeroed fp32 gradient buffer per tensor in dev_grads
 * (the caller writes, not accumulates, unless it wants to accumulate into zeros).
 * GPU-optimised layers evicted during FP are restaged from their HBM master by K1.
 * SH_POST: per-layer Σg² (K3), [world_size>1: NCCL average allreduce], then for a
 * host-optimised layer the D2H gradient offload (PAPER.md:111 step 2) and the CPU
 * Adam dispatch (step 3) that runs while the GPU continues. */
sh_status sh_backward_layer(sh_ctx* ctx, int32_t layer, int32_t phase, void** dev_params,
                            float** dev_grads);

/* Views of the resident set: compute copies (bf16 or fp32) and fp32 grads.  The grads
 * are zeroed at the first forward hook of every step. */
sh_status sh_resident(sh_ctx* ctx, void** dev_params, float** dev_grads);

/* NEXT-3 executors (sh_config.n_executors = K >= 2).  Writes the n_tensors fp32 gradient
 * pointers of executor `executor` (0..K-1) for `layer` -- which must be between its
 * sh_backward_layer PRE and POST -- or for the resident set (layer -1, any time in a step).
 * Executor 0's are the pointers the hooks / sh_resident return; executors >= 1 get
 * engine-owned buffers, zeroed on the compute stream at the PRE (layers) or the first forward
 * hook (resident set).  Contract: every executor's work on a layer is enqueued after its PRE
 * was issued on the compute stream and joined back into the compute stream (an event wait)
 * before the POST; every executor works on an equal share of the batch and computes the
 * gradient of its own micro-batch MEAN loss.  At the POST (sh_step for the resident set) K4
 * computes g = (((g_0 + g_1) + g_2) + ... + g_{K-1}) * fp32(1/K), a fixed order, so results stay
 * bit-identical across windows.  Library-owned; valid until the POST / next sh_step. */
sh_status sh_executor_grads(sh_ctx* ctx, int32_t layer, int32_t executor, float** dev_grads);

/* FP-only pass (NEXT-4: streaming inference of a model larger than HBM, e.g. the teacher of
 * knowledge distillation): call after sh_forward_layer(L-1, SH_POST) instead of
 * the backward hooks.  Nothing is updated, the step counter does not advance and every layer copy
 * in the ring stays valid for the next pass (whose prefetches reuse them). */
sh_status sh_forward_only_end(sh_ctx* ctx);

/* Learning rate for the steps whose backward starts after this call. */
sh_status sh_set_lr(sh_ctx* ctx, double lr);

/* End of step: finalize the global gradient norm in fixed order (K3
 * partials), then one fused multi-tensor AdamW (K2) over layers [0, w) and the
 * resident set writing their new compute copies in place; in clip mode release the
 * CPU Adam tasks with the clip coefficient.  Does not block unless grad_norm_out is
 * non-NULL (then it synchronises and returns ||g||_2). */
sh_status sh_step(sh_ctx* ctx, double* grad_norm_out);

/* ---- window ----------------------------------------------------------------------- */

/* Pure solver of the paper's analytic model P1 (eq. 1a-1d), P2 (eq. 2a-2d) and the
 * window rule of PAPER.md:195, with the eq. 3 / eq. 4 checks reported.  No context,
 * no GPU.  Returns SH_ERR_INVALID for inconsistent profiles. */
sh_status sh_solve_window(const sh_profile* prof, sh_solve_report* report);

/* Solve on the measured warm-up profile (or on `override` when non-NULL) and apply the
 * result between steps (ring grows, never shrinks).  window_out may be NULL. */
sh_status sh_autotune_window(sh_ctx* ctx, const sh_profile* override_profile, int32_t* window_out);

/* Change the window between steps (after sh_step, before the next forward hook). */
sh_status sh_set_window(sh_ctx* ctx, int32_t window);

/* Change the GPU-optimised set size (window) and the ring cap together (ring_slots 0: window+1). */
sh_status sh_set_window_ring(sh_ctx* ctx, int32_t window, int32_t ring_slots);

/* Fill the engine's measured profile (arrays owned by ctx, valid until the next call). */
sh_status sh_get_profile(sh_ctx* ctx, sh_profile* out);

/* ---- inspection ------------------------------------------------------------------- */

/* Blocking copy of one layer's state (layer -1: resident) into host dst, in the caller's
 * tensor order without padding.  Waits for any pending update of that layer. */
sh_status sh_read_layer(sh_ctx* ctx, int32_t layer, int32_t what, void* dst);

sh_status sh_stats(sh_ctx* ctx, sh_stats_t* out);

/* Intervals of the last harvested profiled step (SH_FLAG_PROFILE or warm-up steps); *n_out is
 * the number available (at most cap are written).  Blocks like sh_stats (harvests first). */
sh_status sh_get_trace(sh_ctx* ctx, sh_trace_event* out, int32_t cap, int32_t* n_out);

/* Thread-local message of the last failed call ("" if none). */
const char* sh_last_error(void);

/* ---- NUMA host logic; pure functions of the topology, no CUDA context needed.
 * SH_SYSFS_ROOT (tests) prefixes every sysfs path read by them. */
/* Online nodes: writes up to cap node ids and their CPU counts; returns the node count (>= 1; a
 * host without NUMA sysfs is one node holding every online CPU). */
int32_t sh_numa_topology(int32_t* node_ids, int32_t* n_cpus, int32_t cap);
/* Node INDEX (into sh_numa_topology's order) that host-store unit `unit` (a layer) is placed on
 * under `policy`, -1 = no binding, -2 = interleaved.  gpu_node: the GPU's node index; shared: 1
 * for a data-parallel shared store (AUTO resolves to LOCAL there). */
int32_t sh_numa_plan(int32_t policy, int32_t unit, int32_t n_nodes, int32_t gpu_node, int32_t shared);
/* Node index CPU Adam worker `tid` of n_threads is pinned to (-1: not pinned). */
int32_t sh_numa_worker_node(int32_t policy, int32_t tid, int32_t n_threads, int32_t gpu_node);
/* Node index of a PCI device ("0000:1b:00.0", as cudaDeviceGetPCIBusId prints it); 0 if unknown. */
int32_t sh_numa_node_of_pci(const char* bus_id);
/* Self-check of the placement primitive: mbind(MPOL_BIND) `bytes` of fresh anonymous memory to
 * node id `node_id`, touch it, return the node get_mempolicy reports for its first and last page
 * (-1 if they differ or a syscall failed). */
int32_t sh_numa_bind_check(int32_t node_id, int64_t bytes);

/* NEXT-2 disk probe: write then read `bytes` of a fresh file in dir with the spill tier's own O_DIRECT
 * io_uring transfers (write timed through fdatasync); GB/s each way; *direct = 1 if O_DIRECT was
 * accepted.  The file is unlinked at creation.  No CUDA context needed. */
sh_status sh_spill_probe(const char* dir, int64_t bytes, double* read_gbs, double* write_gbs, int32_t* direct);

int32_t sh_abi_version(void);

/* Number of engine kernel launches (K1, K2, K3, K4, norm finalize) since the library was loaded. */
int64_t sh_kernel_launches(void);

/* Rank 0 of a data-parallel job: fill a 128-byte ncclUniqueId (dlopen'ed libnccl.so.2, the
 * one torch loads) to be broadcast through torch.distributed before sh_init. */
sh_status sh_nccl_get_unique_id(void* out128);

/* ---- op-level entry points (the kernels of the path, for parity tests) -------------
 * All device pointers must be 16-byte aligned and n a multiple of 8.  `stream` is a
 * cudaStream_t (NULL = legacy default).  Asynchronous; errors from the launch only. */

typedef struct {
  float beta1, beta2, omb1, omb2, eps, step_size, sqrt_bc2, decay;
} sh_adam_scalars;

/* Host-side derivation of the per-step fp32 scalars from (lr, t) in double. */
sh_status sh_adam_scalars_for(double lr, double beta1, double beta2, double eps, double weight_decay,
                              int64_t t, sh_adam_scalars* out);

/* K2 on one flat tensor range: elements [0, n_decay) get weight decay, [n_decay, n) not.
 * p, m, v: fp32 in/out; g: fp32 in; out16: bf16 compute copy out (uint16 bits) or NULL;
 * out32: fp32 compute copy out or NULL; coef: device float (clip coefficient) or NULL. */
sh_status sh_op_adamw_gpu(float* p, float* m, float* v, const float* g, uint16_t* out16,
                          float* out32, int64_t n, int64_t n_decay, const sh_adam_scalars* sc,
                          const float* coef, void* stream);

/* The CPU AdamW of the pool on host arrays (same contract as above; coef is a host
 * value, ignored when use_coef == 0).  n_threads <= 0: all cores. */
sh_status sh_op_adamw_cpu(float* p, float* m, float* v, const float* g, uint16_t* out16,
                          int64_t n, int64_t n_decay, const sh_adam_scalars* sc, int32_t use_coef,
                          float coef, int32_t n_threads);

/* K1: dst16[i] = rna_bf16(src[i]) on the device. */
sh_status sh_op_cast_bf16_gpu(const float* src, uint16_t* dst16, int64_t n, void* stream);

/* CPU rna_bf16 (the shadow writer of the CPU Adam). */
sh_status sh_op_cast_bf16_cpu(const float* src, uint16_t* dst16, int64_t n);

/* Split master (host arrays, R25): hi[i] = rna_bf16(p[i]), lo[i] = low 16 bits of bits(p[i]) ... */
sh_status sh_op_master_split_cpu(const float* p, uint16_t* hi, uint16_t* lo, int64_t n);
/* ... and back: p[i] = bits((hi[i] << 16) + sext16(lo[i])). */
sh_status sh_op_master_join_cpu(const uint16_t* hi, const uint16_t* lo, float* p, int64_t n);
/* The CPU AdamW of the pool on a split master (hi, lo in/out; m, v in/out; g in), same contract as
 * sh_op_adamw_cpu: the joined result equals sh_op_adamw_cpu's p bitwise and hi its bf16 output. */
sh_status sh_op_adamw_split_cpu(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t n,
                                int64_t n_decay, const sh_adam_scalars* sc, int32_t use_coef, float coef,
                                int32_t n_threads);

/* K2S (R28): the same split-master AdamW on the GPU (device pointers, no clipping), bitwise
 * sh_op_adamw_split_cpu; n, n_decay multiples of 8, 16-byte aligned pointers; enqueued on `stream`. */
sh_status sh_op_adamw_split_gpu(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t n,
                                int64_t n_decay, const sh_adam_scalars* sc, void* stream);

/* K4 (NEXT-3): dst[i] = (((dst[i] + src[0][i]) + src[1][i]) + ... + src[n_src-1][i]) * inv_k,
 * every op IEEE fp32 round-to-nearest; src is a HOST array of n_src (0..7) device pointers. */
sh_status sh_op_exec_reduce_gpu(float* dst, const float* const* src, int32_t n_src, int64_t n, float inv_k,
                                void* stream);

/* K3: out[0] = Σ g[i]^2 accumulated in fp64 with a fixed reduction tree (deterministic). */
sh_status sh_op_sumsq_gpu(const float* g, int64_t n, double* out_dev, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* SH_H_ */
