// STRONGHOLD working-window offload engine for B200.
//
// Paper mechanism -> this file:
//   pinned per-layer CPU buffers            -> HostStore: one mmap'ed, THP-advised,
//                                                              page-locked block per host layer;
//                                                              bf16: split master hi | lo | m | v (the hi
//                                                              plane IS the compute copy, R25), or
//                                                              fp32 master | m | v [| bf16 shadow];
//                                                              NUMA placement by mbind before first
//                                                              touch (numa.cpp, sh_config.numa_policy)
//   reserved round-robin GPU buffer queue -> ring of w+1 slots, one cudaMalloc,
//                                                              grow-only; param half + grad half
//                                                              (or decoupled from the GPU set, R22)
//   fixed-size buffer, variable layer count  -> sh_config.ring_bytes: variable-capacity
//                                                              slots in one buffer, capacity-filtered
//                                                              Belady (NEXT-4)
//   pre_forward / post_forward (Fig. 3b)      -> sh_forward_layer PRE/POST
//   pre_backward (Fig. 3c)                    -> sh_backward_layer PRE/POST
//   "idle CUDA stream" async copies          -> H2D and D2H copy-engine streams, each
//                                                              owned by an issuer thread; gradients wait
//                                                              in a pool (the ring's grad halves) and
//                                                              are offloaded lowest computed layer
//                                                              first (d2h_pump, R26)
//   concurrent CPU optimizers            -> AdamPool: worker threads, per-layer
//                                                              jobs split into chunks, lowest layer
//                                                              (needed first by the next FP) first
//   first window + embedding updated on GPU  -> K2 over layers [0,w) + resident set
//   warm-up profiling                         -> CUDA events per layer / transfer
//   NCCL data-parallel gradient sync    -> per-layer ncclAllReduce(avg) on a
//                                                              comm stream before the offload
//
// Which slot a fetch lands in: the use sequence of one step is fixed (FP 0..L-1, BP L-1..0), so
// the victim is chosen by farthest next use (Belady) among slots whose occupant is not needed
// before the fetched layer; this reproduces the paper's sliding window (FP: the slot of layer
// i-1 receives layer i+w; BP: the slot of layer i+1 receives layer i-w) and handles the FP/BP
// turn, w = 0 and w = L uniformly.
//
// No host stall on the GPU: PRE/POST only enqueue work and record events.  The single true
// cross-device dependency -- "the prefetch of host layer j for step t must read the parameters
// the CPU Adam produced in step t-1" -- is enforced by the H2D issuer thread waiting on the
// layer's ready counter before it enqueues the copy (this B200 box reports no stream-memop
// support, profiles/r01_probe_box.json, so cuStreamWaitValue32 is not used).
#include <dlfcn.h>
#include <pthread.h>
#include <sched.h>
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <sys/statvfs.h>

#include <cerrno>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <condition_variable>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <functional>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include <nccl.h>

#include "sh_internal.hpp"

namespace sh {
const char* last_error_cstr();
}

using namespace sh;

namespace {

constexpr int64_t kInf = INT64_MAX / 4;
constexpr int64_t kPinned = -1;
constexpr int64_t kCpuChunk = 1 << 18;  // elements per CPU Adam task chunk (~7.5 MB of traffic)

double now_ms() {
  return std::chrono::duration<double, std::milli>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

int64_t align_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// SH_FLAG_DELAY_INJECT: random 0..2 ms host sleeps in the issuers and CPU Adam tasks and random
// GPU spin kernels are NOT used; the host sleeps perturb every cross-thread ordering the engine
// relies on.  Thread-local xorshift, seeded per thread.
void maybe_delay(uint64_t flags) {
  if (!(flags & SH_FLAG_DELAY_INJECT)) return;
  static thread_local uint64_t x = 0x9E3779B97F4A7C15ull ^ (uint64_t)pthread_self();
  x ^= x << 13;
  x ^= x >> 7;
  x ^= x << 17;
  if ((x & 3) == 0) usleep((useconds_t)(x % 2000));
}

double wait_timeout_s() {
  const char* e = getenv("SH_WAIT_TIMEOUT_S");
  return e ? atof(e) : 600.0;
}

// ---- NCCL (dlopen'ed: the process must share torch's libnccl.so.2) ------------------------
struct Nccl {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*CommSplit)(ncclComm_t, int, int, ncclComm_t*, ncclConfig_t*) = nullptr;
  ncclResult_t (*ReduceScatter)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                                cudaStream_t) = nullptr;
  ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
  ncclResult_t (*CommAbort)(ncclComm_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool load() {
    if (h) return true;
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* n : names) {
      h = dlopen(n, RTLD_NOW | RTLD_NOLOAD | RTLD_GLOBAL);
      if (!h) h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
      if (h) break;
    }
    if (!h) return false;
    GetUniqueId = (decltype(GetUniqueId))dlsym(h, "ncclGetUniqueId");
    CommInitRank = (decltype(CommInitRank))dlsym(h, "ncclCommInitRank");
    AllReduce = (decltype(AllReduce))dlsym(h, "ncclAllReduce");
    CommDestroy = (decltype(CommDestroy))dlsym(h, "ncclCommDestroy");
    AllGather = (decltype(AllGather))dlsym(h, "ncclAllGather");
    CommSplit = (decltype(CommSplit))dlsym(h, "ncclCommSplit");
    ReduceScatter = (decltype(ReduceScatter))dlsym(h, "ncclReduceScatter");
    CommGetAsyncError = (decltype(CommGetAsyncError))dlsym(h, "ncclCommGetAsyncError");
    CommAbort = (decltype(CommAbort))dlsym(h, "ncclCommAbort");
    GetErrorString = (decltype(GetErrorString))dlsym(h, "ncclGetErrorString");
    return GetUniqueId && CommInitRank && AllReduce && CommDestroy && GetErrorString && ReduceScatter &&
           AllGather && CommGetAsyncError && CommAbort;
  }
};
Nccl g_nccl;

// ---- FIFO issuer thread (owns one copy stream) --------------------------------------------
class Issuer {
 public:
  void start() { th_ = std::thread([this] { loop(); }); }
  void push(std::function<void()> f) {
    {
      std::lock_guard<std::mutex> g(mu_);
      q_.push_back(std::move(f));
      ++pushed_;
    }
    cv_.notify_one();
  }
  void drain() {  // block until every pushed closure has run
    std::unique_lock<std::mutex> g(mu_);
    cv_done_.wait(g, [&] { return done_ == pushed_; });
  }
  void stop() {
    {
      std::lock_guard<std::mutex> g(mu_);
      stop_ = true;
    }
    cv_.notify_one();
    if (th_.joinable()) th_.join();
  }

 private:
  void loop() {
    for (;;) {
      std::function<void()> f;
      {
        std::unique_lock<std::mutex> g(mu_);
        cv_.wait(g, [&] { return stop_ || !q_.empty(); });
        if (q_.empty()) return;
        f = std::move(q_.front());
        q_.pop_front();
      }
      f();
      {
        std::lock_guard<std::mutex> g(mu_);
        ++done_;
      }
      cv_done_.notify_all();
    }
  }
  std::thread th_;
  std::mutex mu_;
  std::condition_variable cv_, cv_done_;
  std::deque<std::function<void()>> q_;
  int64_t pushed_ = 0, done_ = 0;
  bool stop_ = false;
};

struct ProfSet {  // CUDA timing events of one step (double-buffered by step parity)
  std::vector<cudaEvent_t> fp0, fp1, bp0, bp1, c2g0[2], c2g1[2], g2c0, g2c1, st0, st1, k30, k31, k2l0, k2l1;
  std::vector<std::atomic<uint8_t>> rec_c2g[2], rec_g2c, rec_st;
  std::vector<uint8_t> rec_fp, rec_bp, rec_k3, rec_k2l;
  cudaEvent_t k2a = nullptr, k2b = nullptr, t0 = nullptr;
  bool rec_k2 = false, rec_t0 = false;
  // host-side intervals of this step (CPU Adam jobs, H2D-issuer waits on them), in host ms; t0_host is
  // the host clock when the compute stream passed t0 (a host function right behind the event)
  std::atomic<double> t0_host{0.0};
  std::vector<sh_trace_event> host_iv;  // guarded by sh_ctx::pmu
  bool active = false;
  int64_t step = -1;
  int64_t k2_bytes = 0;
  int k2_launches = 0;
};

}  // namespace

struct GState {
  float* master = nullptr;
  float* m = nullptr;
  float* v = nullptr;
};

struct Job {
  int layer;
  int64_t step;
  double t_first = 0.0;  // host ms when its first chunk was taken (trace)
  // the arrays the update works on: the layer's pinned host block, or (NEXT-2 spilled layer) a pinned
  // staging copy its optimizer state was read into
  float *p = nullptr, *m = nullptr, *v = nullptr;
  uint16_t* sh16 = nullptr;  // bf16 shadow out, or (split master) the hi plane in/out
  uint16_t* lo16 = nullptr;  // split master: the lo plane in/out (then p is unused)
  char* staging = nullptr;
  int landing;
  int64_t lo, hi;  // element range of this rank (whole layer unless the store is shared)
  int64_t n_chunks;
  int64_t next = 0;
  std::atomic<int64_t> done{0};
  sh_adam_scalars sc;
};

// Control block of a shared (multi-process, one box) host store, in /dev/shm.
constexpr int kMaxHostCollRanks = 64;
struct ShmCtl {
  std::atomic<int64_t> magic;
  std::atomic<int64_t> created;    // rank 0 finished creating the layer segments
  std::atomic<int64_t> bar[6];     // monotonic barrier counters
  std::atomic<int64_t> window;     // rank 0's autotuned window (every rank must use the same one)
  std::atomic<int64_t> hc_arrive[kMaxHostCollRanks];  // SH_FLAG_TEST_HOST_COLLECTIVE: per-rank sequence
  std::atomic<int64_t> hc_done[kMaxHostCollRanks];    //   numbers (contribution written / result read)
  std::atomic<int64_t> cnt[1];     // [2L]: cnt[x] slice updates completed (W per step);
                                   //       cnt[L+x] offloads landed (W per step)
};

struct sh_ctx {
  // ---- configuration
  sh_config cfg{};
  int L = 0;
  std::vector<LayerLayout> lay;
  LayerLayout res;
  bool bf16 = true;
  int cb = 2;
  int64_t max_pad = 0;
  int64_t slot_param_bytes = 0, slot_grad_bytes = 0, slot_bytes = 0;
  int w = 0;
  int n_slots = 0;   // slots with bookkeeping (grow-only)
  int ring_alloc = 0;  // slots currently allocated (0 while a regrow failed)
  int n_active = 0;  // slots in use = min(w + 1, ring cap)
  int d = 0;         // prefetch distance = n_active - 1 (the paper's window m when the ring is w+1)
  int ring_cap = 0;  // sh_config.ring_slots / sh_set_window_ring (0: w + 1)
  // NEXT-4 fixed-byte window (sh_config.ring_bytes): variable-capacity slots packed
  // into one buffer of a fixed byte size; empty = fixed-size slots
  std::vector<int64_t> slot_off, slot_cap, slot_pb;  // byte offset, capacity (elements), param-half bytes
  int64_t byte_ring_total = 0;
  bool byte_ring() const { return !slot_off.empty(); }
  int64_t ring_bytes_for(int n) const { return byte_ring() ? byte_ring_total : (int64_t)n * slot_bytes; }
  int64_t slot_param_bytes_of(int s) const { return byte_ring() ? slot_pb[s] : slot_param_bytes; }
  bool k2_layer = true;  // no clipping: a GPU-optimised layer is updated right after its backward
  int ring_for(int w_) const {
    if (byte_ring()) return (int)slot_off.size();  // the whole fixed-size buffer is always in use
    int r = w_ + 1;
    if (k2_layer && ring_cap > 0 && ring_cap < r) r = ring_cap;  // G grads are not pinned: ring may be smaller
    return r;
  }
  int D = 0;         // host landing buffers
  bool clip = false;
  int warmup = 5;
  bool autotune_pending = false;
  int W = 1, rank = 0;

  // ---- streams
  cudaStream_t cs = nullptr, h2d = nullptr, d2h = nullptr, stage = nullptr, comm = nullptr;
  cudaStream_t k3s = nullptr;  // K3 of host layers, beside the D2H copy of the same gradients
  // R28 hybrid update: lo / m / v fetches into HBM staging, K2S, write-backs (one stream each, so a
  // layer's K2S never queues behind the previous layer's write-back)
  cudaStream_t hyb_in = nullptr, hyb_k = nullptr, hyb_out = nullptr;
  std::vector<char*> hyb_stg;  // staging buffers [lo 2n | m 4n | v 4n] of the largest layer
  std::vector<cudaEvent_t> ev_stg_in, ev_stg_k2, ev_stg_free;
  std::vector<int> hyb_stg_of;         // per layer: staging buffer of its current update
  std::vector<int64_t> hyb_issued;     // per layer: step whose staging fetch was issued (-1: none)
  int64_t hyb_rr = 0;
  unsigned int* k2_sched_hyb = nullptr;
  std::atomic<int64_t> hyb_updates{0}, hyb_h2d{0}, hyb_d2h{0};
  ncclComm_t nccl = nullptr;
  ncclComm_t nccl_fetch = nullptr;  // NEXT-1: collectives issued by the H2D issuer thread
  bool slice_fetch = false;
  int64_t cs_max = 0;               // equal slice length (elements) used by the all-gather

  // ---- device memory
  char* ring = nullptr;
  std::vector<GState> g;  // [L]
  float *res_master = nullptr, *res_m = nullptr, *res_v = nullptr, *res_grad = nullptr;
  // NEXT-3 multi-stream executors: executor e >= 1 writes its micro-batch
  // gradients into xgrad[e-1] (layer in BP) / xres[e-1] (resident set); K4 folds them into
  // executor 0's buffers (the engine's own) at the backward POST / sh_step
  int K = 1;
  std::vector<float*> xgrad, xres;
  float* cur_gdst = nullptr;  // executor 0's grad buffer of the layer between backward PRE and POST
  void* res_compute = nullptr;
  double* partials = nullptr;  // [L+1]
  double* scratch_cs = nullptr;
  double* scratch_comm = nullptr;
  double* scratch_d2h = nullptr;
  cudaEvent_t ev_k3_last = nullptr;  // after the K3 of the latest host-layer offload (D2H stream)
  cudaEvent_t ev_res_k3[2] = {nullptr, nullptr}, ev_norm[2] = {nullptr, nullptr};  // by step parity
  int64_t k3_last_gen = 0;            // generation of that offload request
  std::atomic<int64_t> k3_pub{0};     // latest generation whose K3 has been enqueued
  double* norm_dev = nullptr;
  float* coef_dev = nullptr;
  // K2 dynamic-schedule counters (kernels.cu kDyn), one pair per stream K2 runs on; zeroed at init and
  // left zeroed by every launch (null: static schedule, SH_K2_SCHED=static)
  unsigned int* k2_sched_cs = nullptr;
  unsigned int* k2_sched_comm = nullptr;
  int64_t device_bytes = 0;

  // ---- host store: one pinned block per host-optimised layer (allocated when the layer first
  // becomes host-optimised) + one block for the landing ring and scalars
  struct HostBlock {
    char* p = nullptr;
    size_t bytes = 0;
    int fd = -1;  // NEXT-2: >= 0 for a file-backed (spilled, pageable) block
  };
  std::vector<HostBlock> hblocks;  // [L]
  std::vector<HostBlock> hshadow;  // [L] bf16 shadows added after autotune (SH_FLAG_LATE_SHADOW)
  HostBlock hland;
  size_t host_bytes = 0;
  // NUMA placement (numa.cpp): resolved policy, node count, this GPU's node index,
  // per-layer target node (index, numa::kNone / kInterleave), per-worker node, bytes bound
  int numa_policy = SH_NUMA_NONE;
  int numa_nodes = 1;
  int numa_gpu = 0;
  std::vector<int> layer_node;
  std::vector<int> worker_node;
  std::vector<int> slice_node;  // shared store: node index of rank r's slices
  int land_node = -1;
  std::atomic<int64_t> numa_bound{0};
  std::atomic<int> numa_pinned{0};
  // NEXT-2 secondary-storage tier: host-optimised layers beyond the pinned
  // budget live in O_DIRECT files (unlinked at creation) under spill_dir; their fetches go through
  // pinned bounce buffers, their CPU updates through pinned staging copies (no page cache)
  std::string spill_dir;
  int64_t pin_budget = 0;
  size_t spill_bytes = 0;
  int n_spilled = 0;
  std::vector<uint8_t> spilled;  // [L]
  char* bounce[2] = {nullptr, nullptr};
  size_t bounce_bytes = 0;
  cudaEvent_t ev_bounce[2] = {nullptr, nullptr};
  int bounce_rr = 0;  // H2D issuer thread only
  // O_DIRECT spill files: [master | m | v | shadow?] regions, each kAlign-aligned; a spilled layer's
  // CPU update reads master/m/v into a pinned staging buffer (spill_rd thread), updates it there and
  // writes master/m/v/shadow back (spill_wr thread) before the layer counts as updated
  bool spill_direct = false;          // the spill files are O_DIRECT (else the file system refused it)
  std::vector<char*> stg_free, stg_all;
  size_t stg_bytes = 0;
  std::mutex stg_mu;
  std::condition_variable stg_cv;
  std::atomic<int64_t> spill_rd_bytes{0}, spill_wr_bytes{0};
  std::atomic<double> spill_io_ms{0.0};
  bool shadow = false;  // SH_FLAG_BF16_SHADOW: fp32 master + a bf16 shadow in host RAM (14 B/param)
  bool split = false;   // bf16 default: split master, hi plane = the compute copy (12 B/param, R25)
  // shared store (world_size > 1 with shm_name): rank r owns elements [slo[x], shi[x]) of layer x
  bool shared = false;
  // the data-parallel (collective) path: world_size > 1, or SH_FLAG_TEST_DP_PATH at world_size 1
  // (a one-rank NCCL communicator: every all-reduce runs, and is the identity)
  bool dp = false;
  bool no_collective = false;
  bool use_nccl = false;   // the collectives go through NCCL (dp, not a test mode)
  // SH_FLAG_TEST_HOST_COLLECTIVE: the collectives run on the driver thread through a shared host
  // segment, summed in a fixed rank order (several ranks on ONE GPU with different data)
  bool host_coll = false;
  float* hc_seg = nullptr;   // [W][hc_count] contributions, /dev/shm, page-locked
  size_t hc_bytes = 0;
  int64_t hc_count = 0;      // floats per rank
  float* hc_tmp = nullptr;   // private pinned result staging
  int64_t hc_seq = 0;
  bool rs_host = false;      // host layers' gradients are reduce-scattered (shared store: slice r only)
  double* partials_all = nullptr;  // [W][L+1] gathered per-rank partial sums of squares
  std::atomic<int> nccl_aborted{0};
  std::string shm_name;
  ShmCtl* ctl = nullptr;
  size_t ctl_bytes = 0;
  std::vector<int64_t> slo, shi;
  int64_t bar_calls[6] = {0, 0, 0, 0, 0, 0};
  std::vector<float*> h_master, h_m, h_v;
  std::vector<uint16_t*> h_shadow;  // bf16 copy the prefetch moves: the shadow, or the split master's hi plane
  std::vector<uint16_t*> h_lo;      // split master: low 16 bits of the fp32 pattern (R25)
  std::vector<float*> landing;
  float* h_coef = nullptr;  // pinned [2]
  std::vector<uint8_t> registered;

  // ---- ring state (driver thread only, except *_pub / ready / the landing free list)
  std::vector<int> slot_layer, layer_slot;
  std::vector<int64_t> slot_last_use;  // global position of the occupant's latest compute (LRU tie-break)
  int64_t pos_clock = 0;
  std::vector<cudaEvent_t> ev_param_free, ev_grad_done, ev_grad_free, ev_reduced;
  std::vector<cudaEvent_t> ev_k3_buf;  // per pool buffer: after the K3 of the layer it holds (D2H issuer)
  std::vector<int64_t> gradfree_gen, gradfree_waited;  // per gradient-pool buffer (slot index)
  std::unique_ptr<std::atomic<int64_t>[]> gradfree_pub;
  std::vector<cudaEvent_t> ev_arrive;
  std::vector<cudaEvent_t> ev_upd;  // [L] after the latest K2 of a GPU-optimised layer (K1 restage waits)
  // no clipping: GPU-optimised layers write their grads into a small rotation of dedicated HBM
  // buffers (not the ring's grad halves, which may still be queued for offload) consumed by their
  // per-layer K2 on a side stream
  std::vector<float*> gbuf;
  std::vector<cudaEvent_t> ev_gbuf_free, ev_gbuf_ready;
  std::vector<int> gbuf_owner, layer_gbuf;
  int64_t gbuf_rr = 0;
  std::vector<int64_t> arrive_gen, compute_waited;
  std::vector<uint8_t> arrive_by_issuer;
  std::unique_ptr<std::atomic<int64_t>[]> arrive_pub;
  std::unique_ptr<std::atomic<int64_t>[]> ready;  // updates applied to layer j
  // host landing buffers: free list (guarded by smu; a CPU update returns its buffer, the D2H
  // scheduler takes one per offload); landing_owner / last_landing: which layer's grads a buffer holds
  std::deque<int> land_free;  // FIFO: a buffer is reused as late as possible (SH_READ_GRAD diagnostics)
  std::vector<int> landing_owner, last_landing;
  // gradient pool (DESIGN.md §6 "gradient pool"): the grad halves of the ring's slots are a pool of
  // gradient buffers not tied to the slot a layer's parameters sit in -- a layer in BP takes any free
  // one, the D2H scheduler frees it once its offload is issued.  gb_owner[b] = layer holding b (-1:
  // free, guarded by smu); layer_gb[x] = buffer of layer x's last backward
  std::vector<int> gb_owner, layer_gb;
  std::vector<int64_t> gb_free_seq;  // release order (smu): the longest-free buffer is taken first
  int64_t gb_free_ctr = 0;
  struct PendD2H {                 // a host layer's gradients waiting for their offload
    int x, b;
    int64_t step, gen, lo, hi;
    sh_adam_scalars sc;
    void* prof;
    cudaEvent_t ready;
    bool k3_on_d2h, k3_done;
  };
  std::mutex dmu;
  std::deque<PendD2H> pend;        // guarded by dmu, in backward (POST) order
  std::atomic<int64_t> pend_posted{0}, pend_k3{0};
  bool d2h_fifo = false;           // SH_D2H_ORDER=fifo: offload in backward order (A/B of the scheduler)
  float* fp32_stage = nullptr;     // SH_FLAG_FETCH_FP32: fp32 master staging for the K1 cast (h2d stream)
  int64_t gen = 0;
  std::mutex smu;
  std::condition_variable scv;

  // ---- protocol
  enum Phase { IDLE, FP, BP } phase = IDLE;
  int last_layer = -1;
  int last_hook = SH_POST;
  int64_t step = 0;
  int64_t fwd_passes = 0;
  bool registered_all = false;
  std::vector<uint8_t> reg_done;
  bool res_reg = false;
  double lr = 0;
  sh_adam_scalars sc{};
  cudaEvent_t ev_comm_done = nullptr, ev_cs_mark = nullptr;

  // ---- CPU Adam pool
  std::vector<std::thread> workers;
  std::mutex pmu;
  std::condition_variable pcv;
  std::deque<std::unique_ptr<Job>> jobs;
  std::vector<float> coef_of_step;  // clip coefficient per step parity slot
  std::vector<int64_t> coef_step;   // which step the value belongs to
  bool pool_stop = false;
  int n_threads = 0;

  // ---- issuers
  Issuer ih2d, id2h;
  Issuer spill_rd, spill_wr;  // NEXT-2 spill-file reads / write-backs (started with the first spilled layer)
  bool spill_threads = false;

  // ---- profiling
  ProfSet prof[2];
  std::vector<double> p_fp, p_bp, p_c2g, p_g2c, p_stage, p_ogpu, p_ocpu, p_slot, p_gstate;
  std::vector<double> p_c2g_out;  // t_c2g as handed to the solver (after the planned fetch mode)
  std::vector<int64_t> p_slot_i, p_gstate_i;
  std::vector<double> cpu_ms_layer;  // host timing of CPU Adam per layer (last)
  std::vector<sh_trace_event> trace;
  double h2d_overlap = 0, d2h_overlap = 0, last_step_ms = 0, compute_busy_ms = 0;
  double t_async_ms = 0.0;
  int64_t n_async = 0;
  int profiled_steps = 0;

  // ---- stats
  std::atomic<int64_t> h2d_bytes{0}, d2h_bytes{0}, h2d_copies{0}, d2h_copies{0}, stage_launches{0};
  std::atomic<int64_t> cpu_elems{0}, cpu_shadow_elems{0};
  std::atomic<double> cpu_ms{0.0}, cpu_wait_ms{0.0};
  double h2d_busy = 0, d2h_busy = 0;
  int64_t h2d_prof_bytes = 0, d2h_prof_bytes = 0;
  double k2_ms_last = 0, k2_ms_sum = 0, k3_ms_sum = 0;
  int64_t k2_bytes_last = 0, k2_bytes_sum = 0, k2_samples = 0, k3_bytes_sum = 0, k3_samples = 0;
  int64_t k2_layer_launches = 0;
  int k2_launches_last = 0;

  // ---- failure
  std::atomic<int> failed{0};
  std::mutex emu;
  std::string async_err;
  int async_status = SH_OK;

  bool is_g(int x) const { return x < w; }
  // R28 hybrid update: the lowest n_hyb host-optimised layers are updated on the GPU (include/sh.h)
  // while the driver waits for a free gradient buffer (the offloads are the bottleneck), CPU AdamW
  // workers with index >= cpu_throttle pause, leaving host DRAM to the D2H copies (SH_CPU_THROTTLE=T;
  // 0 = off, the default)
  int cpu_throttle = 0;
  std::atomic<int> grad_starved{0};
  int n_hyb = 0;
  bool is_hyb(int x) const { return n_hyb > 0 && x >= w && x < w + n_hyb; }
  char* slot_param(int s) const { return byte_ring() ? ring + slot_off[s] : ring + (int64_t)s * slot_bytes; }
  float* slot_grad(int s) const {
    if (byte_ring()) return reinterpret_cast<float*>(ring + slot_off[s] + slot_pb[s]);
    return reinterpret_cast<float*>(ring + (int64_t)s * slot_bytes + slot_param_bytes);
  }
  int layer_at(int pos) const { return pos < L ? pos : 2 * L - 1 - pos; }
};

namespace {

// ---------------------------------------------------------------------------- failure
void async_fail(sh_ctx* c, int status, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  {
    std::lock_guard<std::mutex> g(c->emu);
    if (c->async_status == SH_OK) {
      c->async_status = status;
      c->async_err = buf;
    }
  }
  c->failed.store(1);
  {
    std::lock_guard<std::mutex> g(c->smu);
  }
  c->scv.notify_all();
  c->pcv.notify_all();
}

sh_status check_failed(sh_ctx* c) {
  if (!c->failed.load()) return SH_OK;
  std::lock_guard<std::mutex> g(c->emu);
  set_error("context failed: %s", c->async_err.c_str());
  return SH_ERR_STATE;
}

#define CKC(c, expr)                                                                     \
  do {                                                                                   \
    cudaError_t e_ = (expr);                                                             \
    if (e_ != cudaSuccess) {                                                             \
      async_fail((c), SH_ERR_CUDA, "%s failed: %s", #expr, cudaGetErrorString(e_));      \
      set_error("%s failed: %s", #expr, cudaGetErrorString(e_));                         \
      return SH_ERR_CUDA;                                                                \
    }                                                                                    \
  } while (0)

#define CKA(c, expr)                                                                     \
  do {                                                                                   \
    cudaError_t e_ = (expr);                                                             \
    if (e_ != cudaSuccess) async_fail((c), SH_ERR_CUDA, "%s: %s", #expr, cudaGetErrorString(e_)); \
  } while (0)

// ---- NCCL health (data parallel).  An asynchronous communicator error (a failed or vanished peer)
// fails the context; a wait that times out while NCCL work may be pending aborts the communicators,
// so their kernels exit instead of spinning on the GPU and the box stays usable.
void nccl_abort(sh_ctx* c, const char* why) {
  if (!c->use_nccl || c->nccl_aborted.exchange(1)) return;
  if (c->nccl_fetch) g_nccl.CommAbort(c->nccl_fetch);
  if (c->nccl) g_nccl.CommAbort(c->nccl);
  async_fail(c, SH_ERR_NCCL, "NCCL communicators aborted: %s", why);
}

// false (context failed) if a communicator reports an asynchronous error.  Never called with smu held.
bool nccl_healthy(sh_ctx* c) {
  if (!c->use_nccl) return true;
  if (c->nccl_aborted.load()) return false;
  for (ncclComm_t m : {c->nccl, c->nccl_fetch}) {
    if (!m) continue;
    ncclResult_t r = ncclSuccess;
    if (g_nccl.CommGetAsyncError(m, &r) != ncclSuccess) continue;
    if (r != ncclSuccess && r != ncclInProgress) {
      char b[256];
      snprintf(b, sizeof(b), "asynchronous error: %s", g_nccl.GetErrorString(r));
      nccl_abort(c, b);
      return false;
    }
  }
  return true;
}

// Wait on the engine state condition (timeout => fail, never hang the box).  With a shared store,
// cross-process progress is only visible by polling; with NCCL the communicators are polled for
// asynchronous errors while waiting.
template <class Pred>
bool state_wait(sh_ctx* c, Pred pred, const char* what, double* waited_ms = nullptr) {
  if (pred()) return true;
  const double t0 = now_ms();
  std::unique_lock<std::mutex> g(c->smu);
  bool ok;
  if (c->shared || c->use_nccl) {
    const double deadline = t0 + 1e3 * wait_timeout_s();
    double next_poll = t0 + 20.0;
    for (;;) {
      if (c->failed.load() || pred()) { ok = true; break; }
      if (now_ms() > deadline) { ok = false; break; }
      if (c->use_nccl && now_ms() > next_poll) {
        g.unlock();
        const bool healthy = nccl_healthy(c);
        g.lock();
        if (!healthy) { ok = true; break; }  // failed: reported below
        next_poll = now_ms() + 20.0;
      }
      c->scv.wait_for(g, c->shared ? std::chrono::microseconds(50) : std::chrono::microseconds(5000));
    }
  } else {
    ok = c->scv.wait_for(g, std::chrono::duration<double>(wait_timeout_s()),
                         [&] { return c->failed.load() || pred(); });
  }
  if (waited_ms) *waited_ms = now_ms() - t0;
  if (!ok) {
    g.unlock();
    char b[256];
    snprintf(b, sizeof(b), "timeout waiting for %s", what);
    nccl_abort(c, b);  // no-op without NCCL
    async_fail(c, SH_ERR_STATE, "%s", b);
    return false;
  }
  return !c->failed.load();
}

// cudaStreamSynchronize, except with NCCL: poll the stream and the communicators, abort on timeout.
sh_status stream_sync(sh_ctx* c, cudaStream_t s) {
  if (!c->use_nccl) {
    CKC(c, cudaStreamSynchronize(s));
    return SH_OK;
  }
  const double deadline = now_ms() + 1e3 * wait_timeout_s();
  for (;;) {
    const cudaError_t e = cudaStreamQuery(s);
    if (e == cudaSuccess) return SH_OK;
    if (e != cudaErrorNotReady) CKC(c, e);
    if (!nccl_healthy(c)) return check_failed(c);
    if (now_ms() > deadline) {
      nccl_abort(c, "stream synchronize timed out");
      return check_failed(c);
    }
    usleep(200);
  }
}

void notify_state(sh_ctx* c) {
  { std::lock_guard<std::mutex> g(c->smu); }
  c->scv.notify_all();
}

// Updates applied to host layer x >= t (all W slices when the store is shared)?
bool ready_at_least(const sh_ctx* c, int x, int64_t t) {
  if (c->shared) return c->ctl->cnt[x].load(std::memory_order_acquire) >= (int64_t)c->W * t;
  return c->ready[x].load(std::memory_order_acquire) >= t;
}

// Cross-process barrier on the shared control block (polling).
bool shm_barrier(sh_ctx* c, int id, const char* what) {
  if (!c->shared) return true;
  const int64_t target = (int64_t)c->W * (++c->bar_calls[id]);
  c->ctl->bar[id].fetch_add(1);
  return state_wait(c, [&] { return c->ctl->bar[id].load() >= target; }, what);
}

// ---------------------------------------------------------------------------- host store
void* host_alloc(size_t bytes) {
  void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (p == MAP_FAILED) return nullptr;
  madvise(p, bytes, MADV_HUGEPAGE);
  return p;
}

// first touch in parallel (pages land on the toucher's node; THP => 2 MiB pages)
void parallel_touch(char* p, size_t bytes, int threads) {
  const size_t chunk = align_up((int64_t)(bytes / std::max(threads, 1) + 1), 1 << 21);
  std::vector<std::thread> ts;
  for (size_t off = 0; off < bytes; off += chunk) {
    const size_t n = std::min(chunk, bytes - off);
    ts.emplace_back([=] { std::memset(p + off, 0, n); });
  }
  for (auto& t : ts) t.join();
}

int64_t mem_available_bytes() {
  FILE* f = fopen("/proc/meminfo", "r");
  if (!f) return INT64_MAX;
  char key[64];
  long long kb = 0;
  char unit[16];
  int64_t avail = INT64_MAX;
  while (fscanf(f, "%63s %lld %15s", key, &kb, unit) == 3)
    if (strcmp(key, "MemAvailable:") == 0) {
      avail = (int64_t)kb * 1024;
      break;
    }
  fclose(f);
  return avail;
}

// mmap + THP advice + parallel first touch + cudaHostRegister.  Refuses (instead of letting the
// kernel OOM-kill the process) when the block would leave less than SH_HOST_MARGIN_GB free.
sh_status host_block_alloc(size_t bytes, int threads, char** out, int node = numa::kNone,
                           std::atomic<int64_t>* bound = nullptr) {
  *out = nullptr;
  const char* mg = getenv("SH_HOST_MARGIN_GB");
  const int64_t margin = (int64_t)((mg ? atof(mg) : 3.0) * (1ll << 30));
  const int64_t avail = mem_available_bytes();
  if ((int64_t)bytes + margin > avail) {
    set_error("host store: %lld B requested, %lld B available (margin %lld B)", (long long)bytes,
              (long long)avail, (long long)margin);
    return SH_ERR_OOM_HOST;
  }
  char* p = static_cast<char*>(host_alloc(bytes));
  if (!p) {
    set_error("host store: mmap of %lld B failed", (long long)bytes);
    return SH_ERR_OOM_HOST;
  }
  // NUMA placement before the first touch (a no-op on a single-node host)
  if (node != numa::kNone && numa::bind_range(p, bytes, node) && bound) bound->fetch_add((int64_t)bytes);
  parallel_touch(p, bytes, threads);
  if (cudaHostRegister(p, bytes, cudaHostRegisterPortable) != cudaSuccess) {
    cudaGetLastError();
    munmap(p, bytes);
    set_error("host store: cudaHostRegister of %lld B failed (memlock?)", (long long)bytes);
    return SH_ERR_OOM_HOST;
  }
  *out = p;
  return SH_OK;
}

void host_block_free(char* p, size_t bytes) {
  if (!p) return;
  cudaHostUnregister(p);
  munmap(p, bytes);
}

// ---------------------------------------------------------------------------- CPU Adam pool
void host_interval(sh_ctx* c, int kind, int layer, int64_t step, double t0, double t1);

// ---- NEXT-2 spill files (O_DIRECT): region k of layer x (0 master, 1 m, 2 v, 3 bf16 shadow) starts at
// k * sp_rb(x); every region length and offset is a multiple of spill::kAlign
int64_t sp_rb(const sh_ctx* c, int x) { return align_up(4 * c->lay[x].n_pad, (int64_t)spill::kAlign); }
int64_t sp_sb(const sh_ctx* c, int x) {
  return c->shadow ? align_up(2 * c->lay[x].n_pad, (int64_t)spill::kAlign) : 0;
}
int64_t sp_file_bytes(const sh_ctx* c, int x) { return 3 * sp_rb(c, x) + sp_sb(c, x); }
bool has_shadow(const sh_ctx* c, int x) {
  return c->h_shadow[x] != nullptr || (c->spilled[x] && (c->shadow || c->split));
}
// (a split-master spill file holds [hi | lo] in region 0: the fetch reads its first 2n bytes)

// Blocking O_DIRECT transfer of `bytes` (rounded up to kAlign) between buf and layer x's spill file at
// byte offset off.  Any thread; failures fail the context.
sh_status spill_file_io(sh_ctx* c, bool write, int x, void* buf, int64_t bytes, int64_t off = 0) {
  const double t0 = now_ms();
  const int64_t n = align_up(bytes, (int64_t)spill::kAlign);
  const int r = spill::transfer(write, c->hblocks[x].fd, buf, (size_t)n, off);
  if (r != 0) {
    async_fail(c, SH_ERR_OOM_HOST, "spill tier: %s of %lld B (layer %d): %s", write ? "write" : "read",
               (long long)n, x, strerror(-r));
    set_error("spill tier: %s of layer %d failed: %s", write ? "write" : "read", x, strerror(-r));
    return SH_ERR_OOM_HOST;
  }
  (write ? c->spill_wr_bytes : c->spill_rd_bytes).fetch_add(n);
  const double dt = now_ms() - t0;
  double cur = c->spill_io_ms.load();
  while (!c->spill_io_ms.compare_exchange_weak(cur, cur + dt)) {
  }
  return SH_OK;
}

char* acquire_staging(sh_ctx* c) {
  std::unique_lock<std::mutex> g(c->stg_mu);
  const bool ok = c->stg_cv.wait_for(g, std::chrono::duration<double>(wait_timeout_s()),
                                     [&] { return !c->stg_free.empty() || c->failed.load(); });
  if (!ok) {
    g.unlock();
    async_fail(c, SH_ERR_STATE, "timeout waiting for a spill staging buffer");
    return nullptr;
  }
  if (c->failed.load()) return nullptr;
  char* p = c->stg_free.back();
  c->stg_free.pop_back();
  return p;
}

void release_staging(sh_ctx* c, char* p) {
  {
    std::lock_guard<std::mutex> g(c->stg_mu);
    c->stg_free.push_back(p);
  }
  c->stg_cv.notify_all();
}

// The update of `layer` for step `step` is visible to the prefetches (and to the other ranks).
void mark_updated(sh_ctx* c, int layer, int64_t step) {
  c->ready[layer].store(step + 1, std::memory_order_release);
  if (c->shared) c->ctl->cnt[layer].fetch_add(1, std::memory_order_release);
  notify_state(c);
}

void finish_job(sh_ctx* c, Job* j) {
  // landing buffer first, readiness last: sync_all (and so grow_landing, which rebuilds the landing
  // free list) returns once every layer is ready, so no worker may still be about to return a buffer
  {
    std::lock_guard<std::mutex> g(c->smu);
    c->land_free.push_back(j->landing);
  }
  c->scv.notify_all();
  if (j->staging) {
    // spilled layer: updated in its staging copy; it counts as updated once master / m / v / shadow
    // are back in the file (the next fetch reads the file)
    const int x = j->layer;
    const int64_t step = j->step;
    char* stg = j->staging;
    c->spill_wr.push([c, x, step, stg] {
      if (spill_file_io(c, true, x, stg, sp_file_bytes(c, x)) != SH_OK) return;
      release_staging(c, stg);
      mark_updated(c, x, step);
    });
    return;
  }
  mark_updated(c, j->layer, j->step);
}

void worker_loop(sh_ctx* c, int tid) {
  const int my_node = c->worker_node.empty() ? numa::kNone : c->worker_node[tid];
  if (my_node != numa::kNone && numa::pin_thread(my_node)) c->numa_pinned.fetch_add(1);
  // SPLIT: prefer the layers placed on this worker's node (local DRAM); take others only when
  // none of those is eligible, so no worker idles while work is queued
  auto local = [&](const Job* jp) { return my_node < 0 || c->layer_node[jp->layer] == my_node; };
  for (;;) {
    Job* job = nullptr;
    int64_t chunk = -1;
    float coef = 1.0f;
    {
      std::unique_lock<std::mutex> g(c->pmu);
      // shared store: a slice may only be rewritten once every rank's gradients of the layer have
      // landed (then no rank can still be fetching this step's parameters of the layer for its
      // backward).  A real all-reduce implies it; SH_FLAG_TEST_NO_COLLECTIVE relies on it.
      auto eligible = [&](const Job* jp) {
        if (jp->next >= jp->n_chunks) return false;
        if (c->clip && c->coef_step[jp->step & 1] != jp->step) return false;
        if (c->shared && c->ctl->cnt[c->L + jp->layer].load(std::memory_order_acquire) < (int64_t)c->W * (jp->step + 1))
          return false;
        return true;
      };
      auto any = [&] {
        if (c->pool_stop || c->failed.load()) return true;
        for (auto& jp : c->jobs)
          if (eligible(jp.get())) return true;
        return false;
      };
      if (c->cpu_throttle > 0 && tid >= c->cpu_throttle)
        while (c->grad_starved.load() && !c->pool_stop && !c->failed.load())
          c->pcv.wait_for(g, std::chrono::microseconds(200));
      if (c->shared) {
        while (!any()) c->pcv.wait_for(g, std::chrono::microseconds(100));
      } else {
        c->pcv.wait(g, any);
      }
      if (c->pool_stop || c->failed.load()) return;
      // lowest layer first: it is prefetched first by the next FP (eq. 3)
      for (int pass = 0; pass < 2 && !job; ++pass)
        for (auto& jp : c->jobs) {
          if (!eligible(jp.get()) || (pass == 0 && !local(jp.get()))) continue;
          if (!job || jp->step < job->step || (jp->step == job->step && jp->layer < job->layer))
            job = jp.get();
        }
      if (job->next == 0) job->t_first = now_ms();
      chunk = job->next++;
      if (c->clip) coef = c->coef_of_step[job->step & 1];
    }
    maybe_delay(c->cfg.flags);
    const double t0 = now_ms();
    const int x = job->layer;
    const LayerLayout& Lx = c->lay[x];
    const int64_t b = job->lo + chunk * kCpuChunk, e = std::min(job->hi, b + kCpuChunk);
    if (job->lo16)
      cpu::adamw_range_split(job->sh16, job->lo16, job->m, job->v, c->landing[job->landing], b, e, Lx.n_decay,
                             job->sc, c->clip, coef);
    else
      cpu::adamw_range(job->p, job->m, job->v, c->landing[job->landing], job->sh16, b, e, Lx.n_decay, job->sc,
                       c->clip, coef);
    const double dt = now_ms() - t0;
    double cur = c->cpu_ms.load();
    while (!c->cpu_ms.compare_exchange_weak(cur, cur + dt)) {
    }
    c->cpu_elems.fetch_add(e - b);
    if (job->sh16 && !job->lo16) c->cpu_shadow_elems.fetch_add(e - b);
    if (job->done.fetch_add(1) + 1 == job->n_chunks) {
      const double t_end = now_ms();
      finish_job(c, job);
      std::lock_guard<std::mutex> g(c->pmu);
      host_interval(c, 8, job->layer, job->step, job->t_first, t_end);
      for (auto it = c->jobs.begin(); it != c->jobs.end(); ++it)
        if (it->get() == job) {
          c->jobs.erase(it);
          break;
        }
    }
  }
}

struct Landed {
  sh_ctx* c;
  int layer;
  int64_t step;
  int landing;
  sh_adam_scalars sc;
};

void CUDART_CB landed_cb(void* arg) {  // runs on a CUDA driver thread: no CUDA calls here
  std::unique_ptr<Landed> L(static_cast<Landed*>(arg));
  sh_ctx* c = L->c;
  if (c->shared) c->ctl->cnt[c->L + L->layer].fetch_add(1, std::memory_order_release);
  auto j = std::make_unique<Job>();
  j->layer = L->layer;
  j->step = L->step;
  j->landing = L->landing;
  j->lo = c->slo[L->layer];
  j->hi = c->shi[L->layer];
  j->n_chunks = (j->hi - j->lo + kCpuChunk - 1) / kCpuChunk;
  j->sc = L->sc;
  const int x = L->layer;
  if (c->spilled[x]) {
    // NEXT-2: the spill-read thread reads master / m / v into a pinned staging buffer, then queues the
    // update on it ("asynchronous bulk read/write requests")
    Job* raw = j.release();
    c->spill_rd.push([c, raw, x] {
      std::unique_ptr<Job> jb(raw);
      char* stg = acquire_staging(c);
      if (!stg) return;
      if (spill_file_io(c, false, x, stg, 3 * sp_rb(c, x)) != SH_OK) {
        release_staging(c, stg);
        return;
      }
      const int64_t rb = sp_rb(c, x);
      jb->staging = stg;
      jb->p = reinterpret_cast<float*>(stg);
      jb->m = reinterpret_cast<float*>(stg + rb);
      jb->v = reinterpret_cast<float*>(stg + 2 * rb);
      jb->sh16 = c->shadow ? reinterpret_cast<uint16_t*>(stg + 3 * rb) : nullptr;
      if (c->split) {  // region 0 = [hi | lo]
        jb->p = nullptr;
        jb->sh16 = reinterpret_cast<uint16_t*>(stg);
        jb->lo16 = reinterpret_cast<uint16_t*>(stg) + c->lay[x].n_pad;
      }
      {
        std::lock_guard<std::mutex> g(c->pmu);
        c->jobs.push_back(std::move(jb));
      }
      c->pcv.notify_all();
    });
    return;
  }
  j->p = c->h_master[x];
  j->m = c->h_m[x];
  j->v = c->h_v[x];
  j->sh16 = c->h_shadow[x];
  j->lo16 = c->h_lo[x];
  if ((c->cfg.flags & SH_FLAG_SYNC_CPU) && !c->clip && !c->shared) {  // debug: inline, single-threaded
    Job* jp = j.get();
    const float coef = 1.0f;
    if (jp->lo16)
      cpu::adamw_range_split(jp->sh16, jp->lo16, jp->m, jp->v, c->landing[jp->landing], jp->lo, jp->hi,
                             c->lay[jp->layer].n_decay, jp->sc, c->clip, coef);
    else
      cpu::adamw_range(jp->p, jp->m, jp->v, c->landing[jp->landing], jp->sh16, jp->lo, jp->hi,
                       c->lay[jp->layer].n_decay, jp->sc, c->clip, coef);
    finish_job(c, jp);
    return;
  }
  {
    std::lock_guard<std::mutex> g(c->pmu);
    c->jobs.push_back(std::move(j));
  }
  c->pcv.notify_all();
}

struct CoefMsg {
  sh_ctx* c;
  int64_t step;
};
void CUDART_CB coef_cb(void* arg) {
  std::unique_ptr<CoefMsg> m(static_cast<CoefMsg*>(arg));
  sh_ctx* c = m->c;
  {
    std::lock_guard<std::mutex> g(c->pmu);
    c->coef_of_step[m->step & 1] = c->h_coef[m->step & 1];
    c->coef_step[m->step & 1] = m->step;
  }
  c->pcv.notify_all();
}

// ---------------------------------------------------------------------------- profiling
sh_status prof_alloc(sh_ctx* c, ProfSet& P) {
  auto mk = [&](std::vector<cudaEvent_t>& v) -> cudaError_t {
    v.assign(c->L, nullptr);
    for (auto& e : v) {
      cudaError_t r = cudaEventCreate(&e);
      if (r != cudaSuccess) return r;
    }
    return cudaSuccess;
  };
  cudaError_t r = cudaSuccess;
  for (auto* v : {&P.fp0, &P.fp1, &P.bp0, &P.bp1, &P.c2g0[0], &P.c2g1[0], &P.c2g0[1], &P.c2g1[1],
                  &P.g2c0, &P.g2c1, &P.st0, &P.st1, &P.k30, &P.k31, &P.k2l0, &P.k2l1})
    if (r == cudaSuccess) r = mk(*v);
  if (r == cudaSuccess) r = cudaEventCreate(&P.k2a);
  if (r == cudaSuccess) r = cudaEventCreate(&P.k2b);
  if (r == cudaSuccess) r = cudaEventCreate(&P.t0);
  if (r != cudaSuccess) {
    set_error("cudaEventCreate: %s", cudaGetErrorString(r));
    return SH_ERR_CUDA;
  }
  P.rec_c2g[0] = std::vector<std::atomic<uint8_t>>(c->L);
  P.rec_c2g[1] = std::vector<std::atomic<uint8_t>>(c->L);
  P.rec_g2c = std::vector<std::atomic<uint8_t>>(c->L);
  P.rec_st = std::vector<std::atomic<uint8_t>>(c->L);
  P.rec_fp.assign(c->L, 0);
  P.rec_bp.assign(c->L, 0);
  P.rec_k3.assign(c->L, 0);
  P.rec_k2l.assign(c->L, 0);
  return SH_OK;
}

void prof_reset(sh_ctx* c, ProfSet& P, int64_t step) {
  for (int i = 0; i < c->L; ++i) {
    P.rec_c2g[0][i] = 0;
    P.rec_c2g[1][i] = 0;
    P.rec_g2c[i] = 0;
    P.rec_st[i] = 0;
    P.rec_fp[i] = 0;
    P.rec_bp[i] = 0;
    P.rec_k3[i] = 0;
    P.rec_k2l[i] = 0;
  }
  P.rec_k2 = false;
  P.rec_t0 = false;
  P.t0_host.store(0.0);
  {
    std::lock_guard<std::mutex> g(c->pmu);
    P.host_iv.clear();
  }
  P.active = true;
  P.step = step;
}

void CUDART_CB t0_cb(void* arg) { static_cast<ProfSet*>(arg)->t0_host.store(now_ms()); }

// A host-side interval of step `step` (under pmu): CPU Adam job (kind 8) or H2D wait on it (kind 9).
void host_interval(sh_ctx* c, int kind, int layer, int64_t step, double t0, double t1) {
  ProfSet& P = c->prof[step & 1];
  if (P.active && P.step == step) P.host_iv.push_back(sh_trace_event{kind, layer, t0, t1});
}

float ev_ms(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0;
  if (cudaEventSynchronize(b) != cudaSuccess) return 0;
  if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) return 0;
  return ms;
}

float ev_at(cudaEvent_t t0, cudaEvent_t e) {
  float ms = 0;
  if (cudaEventSynchronize(e) != cudaSuccess) return 0;
  if (cudaEventElapsedTime(&ms, t0, e) != cudaSuccess) return 0;
  return ms;
}

double union_overlap(std::vector<std::pair<double, double>> comp, const std::vector<std::pair<double, double>>& cp,
                     double* copy_total) {
  std::sort(comp.begin(), comp.end());
  std::vector<std::pair<double, double>> u;
  for (auto& iv : comp) {
    if (!u.empty() && iv.first <= u.back().second) u.back().second = std::max(u.back().second, iv.second);
    else u.push_back(iv);
  }
  double ov = 0, tot = 0;
  for (auto& c : cp) {
    tot += c.second - c.first;
    for (auto& v : u) ov += std::max(0.0, std::min(c.second, v.second) - std::max(c.first, v.first));
  }
  *copy_total = tot;
  return ov;
}

void build_trace(sh_ctx* c, ProfSet& P) {
  if (!P.rec_t0) return;
  c->trace.clear();
  auto add = [&](int kind, int layer, cudaEvent_t a, cudaEvent_t b) {
    c->trace.push_back(sh_trace_event{kind, layer, ev_at(P.t0, a), ev_at(P.t0, b)});
  };
  for (int i = 0; i < c->L; ++i) {
    if (P.rec_fp[i]) add(0, i, P.fp0[i], P.fp1[i]);
    if (P.rec_bp[i]) add(1, i, P.bp0[i], P.bp1[i]);
    for (int ph = 0; ph < 2; ++ph)
      if (P.rec_c2g[ph][i]) add(2 + ph, i, P.c2g0[ph][i], P.c2g1[ph][i]);
    if (P.rec_g2c[i]) add(4, i, P.g2c0[i], P.g2c1[i]);
    if (P.rec_st[i]) add(5, i, P.st0[i], P.st1[i]);
    if (P.rec_k3[i]) add(6, i, P.k30[i], P.k31[i]);
    if (P.rec_k2l[i]) add(7, i, P.k2l0[i], P.k2l1[i]);
  }
  if (P.rec_k2) add(7, -1, P.k2a, P.k2b);
  if (P.t0_host.load() > 0) {
    std::lock_guard<std::mutex> g(c->pmu);
    for (const auto& e : P.host_iv)
      c->trace.push_back(sh_trace_event{e.kind, e.layer, e.start_ms - P.t0_host.load(), e.end_ms - P.t0_host.load()});
  }
  std::vector<std::pair<double, double>> comp, h2d, d2h;
  double end = 0;
  for (auto& e : c->trace) {
    if (e.kind <= 7) end = std::max(end, e.end_ms);
    if (e.kind <= 1) comp.emplace_back(e.start_ms, e.end_ms);
    if (e.kind == 2 || e.kind == 3) h2d.emplace_back(e.start_ms, e.end_ms);
    if (e.kind == 4) d2h.emplace_back(e.start_ms, e.end_ms);
  }
  double th = 0, td = 0;
  const double oh = union_overlap(comp, h2d, &th), od = union_overlap(comp, d2h, &td);
  c->h2d_overlap = th > 0 ? oh / th : 0;
  c->d2h_overlap = td > 0 ? od / td : 0;
  c->last_step_ms = P.rec_k2 ? ev_at(P.t0, P.k2b) : end;
  // compute-stream busy time: union of the layer compute intervals and the K2 launches on it
  // (the step-end K2 and, single GPU, the per-layer K2); the rest of the step is stall
  std::vector<std::pair<double, double>> busy = comp;
  for (auto& e : c->trace)
    if (e.kind == 7) busy.emplace_back(e.start_ms, e.end_ms);
  double tb = 0;
  const double whole = union_overlap(busy, {{0.0, std::max(end, c->last_step_ms)}}, &tb);
  c->compute_busy_ms = whole;
}

// Read the events of a finished profiled step into the profile arrays and the stats.
void prof_harvest(sh_ctx* c, ProfSet& P) {
  if (!P.active) return;
  P.active = false;
  build_trace(c, P);
  const int L = c->L;
  for (int i = 0; i < L; ++i) {
    if (P.rec_fp[i]) c->p_fp[i] = ev_ms(P.fp0[i], P.fp1[i]);
    if (P.rec_bp[i]) c->p_bp[i] = ev_ms(P.bp0[i], P.bp1[i]);
    for (int ph = 0; ph < 2; ++ph)
      if (P.rec_c2g[ph][i]) {
        const double ms = ev_ms(P.c2g0[ph][i], P.c2g1[ph][i]);
        c->p_c2g[i] = ms;
        c->h2d_busy += ms;
        c->h2d_prof_bytes += (int64_t)((c->bf16 && !has_shadow(c, i)) ? 4 : c->cb) *
                             (c->slice_fetch && c->use_nccl ? c->shi[i] - c->slo[i] : c->lay[i].n_pad);
      }
    if (P.rec_g2c[i]) {
      const double ms = ev_ms(P.g2c0[i], P.g2c1[i]);
      c->p_g2c[i] = ms;
      c->d2h_busy += ms;
      c->d2h_prof_bytes += 4 * (c->shi[i] - c->slo[i]);
    }
    if (P.rec_st[i]) c->p_stage[i] = ev_ms(P.st0[i], P.st1[i]);
    if (P.rec_k2l[i]) {
      const double ms = ev_ms(P.k2l0[i], P.k2l1[i]);
      c->p_ogpu[i] = ms;
      c->k2_ms_sum += ms;
      c->k2_bytes_sum += (c->bf16 ? 30 : 32) * c->lay[i].n_pad;
      c->k2_layer_launches++;
    }
    if (P.rec_k3[i]) {
      c->k3_ms_sum += ev_ms(P.k30[i], P.k31[i]);
      c->k3_bytes_sum += 4 * c->lay[i].n_pad;
      c->k3_samples++;
    }
  }
  if (P.rec_k2) {
    c->k2_ms_last = ev_ms(P.k2a, P.k2b);
    c->k2_bytes_last = P.k2_bytes;
    c->k2_launches_last = P.k2_launches;
    c->k2_ms_sum += c->k2_ms_last;
    c->k2_bytes_sum += P.k2_bytes;
    c->k2_samples++;
    // apportion K2 time to layers by bytes (one fused launch covers all of them)
    double tot = 0;
    for (int i = 0; i < L; ++i) tot += c->lay[i].n_pad;
    if (!c->k2_layer)
      for (int i = 0; i < L; ++i)
        c->p_ogpu[i] = P.k2_bytes > 0 ? c->k2_ms_last * (30.0 * c->lay[i].n_pad) / P.k2_bytes : 0.0;
  }
  c->profiled_steps++;
}

bool step_profiled(sh_ctx* c, int64_t step) {
  return (c->cfg.flags & SH_FLAG_PROFILE) || step < c->warmup || c->autotune_pending;
}

ProfSet* cur_prof(sh_ctx* c) {
  ProfSet& P = c->prof[c->step & 1];
  return (P.active && P.step == c->step) ? &P : nullptr;
}

// ---------------------------------------------------------------------------- ring logic
int64_t next_use(const sh_ctx* c, int x, int cur) {
  if (x >= cur) return x;  // FP use still ahead
  const int b = 2 * c->L - 1 - x;
  if (b >= cur) return b;  // BP use still ahead
  // after its backward: a host copy goes stale; a GPU-optimised layer's copy was updated in place by
  // its per-layer K2 (valid for the next step's FP) or, in clip mode, its grads wait for sh_step's K2
  // (a hybrid layer's copy was updated in place by its K2S: valid for the next step's FP, like a G layer's)
  if (!c->is_g(x)) return c->is_hyb(x) ? 2 * (int64_t)c->L + x : kInf;
  return c->k2_layer ? 2 * (int64_t)c->L + x : kPinned;
}

sh_status issue_fetch(sh_ctx* c, int y, int s, int pos) {
  if (c->cfg.flags & SH_FLAG_ABLATE_ALLOC) {
    // ablation (Fig. 14 "memory management"): what per-layer buffers from the CUDA
    // allocator would cost -- a cudaMalloc / cudaFree pair per prefetch; cudaFree synchronises the
    // device, so the driver cannot run ahead of the GPU (data placement is unchanged)
    void* tmp = nullptr;
    CKC(c, cudaMalloc(&tmp, c->slot_bytes));
    CKC(c, cudaFree(tmp));
  }
  const int old = c->slot_layer[s];
  if (old >= 0) c->layer_slot[old] = -1;
  c->slot_layer[s] = y;
  c->layer_slot[y] = s;
  const int64_t gen = ++c->gen;
  c->arrive_gen[y] = gen;
  char* dst = c->slot_param(s);
  const int64_t n = c->lay[y].n_pad;
  const bool poison = c->cfg.flags & SH_FLAG_POISON;
  ProfSet* P = cur_prof(c);
  const int ph = pos < c->L ? 0 : 1;
  if (c->is_g(y)) {
    // K1 restage from the HBM master (GPU-optimised layer evicted earlier): after the victim slot is
    // free AND after the layer's latest K2 (its master may have been written on another stream or
    // after the victim's release)
    CKC(c, cudaStreamWaitEvent(c->stage, c->ev_param_free[s], 0));
    CKC(c, cudaStreamWaitEvent(c->stage, c->ev_upd[y], 0));
    if (poison) CKC(c, cudaMemsetAsync(dst, 0xff, c->slot_param_bytes_of(s), c->stage));
    if (P) CKC(c, cudaEventRecord(P->st0[y], c->stage));
    if (c->bf16)
      CKC(c, kern::cast_bf16(c->g[y].master, reinterpret_cast<uint16_t*>(dst), n, c->stage));
    else
      CKC(c, cudaMemcpyAsync(dst, c->g[y].master, 4 * n, cudaMemcpyDeviceToDevice, c->stage));
    if (P) {
      CKC(c, cudaEventRecord(P->st1[y], c->stage));
      P->rec_st[y] = 1;
    }
    CKC(c, cudaEventRecord(c->ev_arrive[y], c->stage));
    c->arrive_by_issuer[y] = 0;
    c->arrive_pub[y].store(gen);
    c->stage_launches++;
    return SH_OK;
  }
  c->arrive_by_issuer[y] = 1;
  const int64_t need = c->step;
  // bf16 mode fetches the bf16 shadow; fp32 mode the master; SH_FLAG_FETCH_FP32 fetches the fp32
  // master into the slot's (idle) grad half and K1 casts it into the param half on the H2D stream
  const bool cast = c->bf16 && !has_shadow(c, y);
  const void* src = c->h_shadow[y] ? (const void*)c->h_shadow[y] : (const void*)c->h_master[y];  // null: spilled
  const int64_t eb = cast ? 4 : (int64_t)c->cb;  // fetched bytes per element
  const int64_t bytes = eb * n;
  // NEXT-1 slice fetch: this rank's slice over PCIe, the rest over NVLink (in-place all-gather)
  const bool slice = c->slice_fetch;
  const int64_t slo = c->slo[y], shi = c->shi[y];
  const int64_t cs = align_up((n + c->W - 1) / c->W, kPad);
  cudaEvent_t pf = c->ev_param_free[s];
  float* stage_buf = c->fp32_stage;  // one buffer: the copy into it and the K1 cast out of it are both on the h2d stream
  const int64_t pbytes = c->slot_param_bytes_of(s);
  c->ih2d.push([c, y, need, src, dst, bytes, pf, gen, poison, P, ph, cast, stage_buf, n, eb, slice, slo, shi, cs,
                pbytes] {
    maybe_delay(c->cfg.flags);
    double waited = 0;
    if (!state_wait(c, [&] { return ready_at_least(c, y, need); }, "CPU Adam of a layer to prefetch", &waited)) {
      c->arrive_pub[y].store(kInf);
      notify_state(c);
      return;
    }
    if (waited > 0) {
      double cur = c->cpu_wait_ms.load();
      while (!c->cpu_wait_ms.compare_exchange_weak(cur, cur + waited)) {
      }
      const double t1 = now_ms();
      std::lock_guard<std::mutex> g(c->pmu);
      host_interval(c, 9, y, need, t1 - waited, t1);  // waiting for the update of step need-1
    }
    CKA(c, cudaStreamWaitEvent(c->h2d, pf, 0));
    if (poison) CKA(c, cudaMemsetAsync(dst, 0xff, pbytes, c->h2d));
    char* buf = cast ? reinterpret_cast<char*>(stage_buf) : dst;
    const char* hsrc = static_cast<const char*>(src);
    if (c->spilled[y]) {
      // NEXT-2: O_DIRECT read of the layer's fetch region (bf16 shadow, else fp32 master) from its
      // spill file straight into a pinned bounce buffer (io_uring, no page cache; overlaps the
      // previous layer's H2D from the other buffer) -> async H2D
      const int k = c->bounce_rr++ & 1;
      CKA(c, cudaEventSynchronize(c->ev_bounce[k]));  // its previous H2D has finished
      // the shadow region; else the master, or a split master's hi plane, both at 0
      const int64_t off = c->shadow ? 3 * sp_rb(c, y) : 0;
      if (spill_file_io(c, false, y, c->bounce[k], bytes, off) != SH_OK) {
        c->arrive_pub[y].store(kInf);
        notify_state(c);
        return;
      }
      hsrc = c->bounce[k];
    }
    if (P) CKA(c, cudaEventRecord(P->c2g0[ph][y], c->h2d));
    if (!slice) {
      CKA(c, cudaMemcpyAsync(buf, hsrc, bytes, cudaMemcpyHostToDevice, c->h2d));
      if (c->spilled[y]) CKA(c, cudaEventRecord(c->ev_bounce[(c->bounce_rr - 1) & 1], c->h2d));
    } else if (shi > slo) {
      CKA(c, cudaMemcpyAsync(buf + eb * slo, hsrc + eb * slo, eb * (shi - slo), cudaMemcpyHostToDevice, c->h2d));
    }
    if (P) {
      CKA(c, cudaEventRecord(P->c2g1[ph][y], c->h2d));
      P->rec_c2g[ph][y] = 1;
    }
    if (slice) {
      if (c->use_nccl) {  // every rank holds slice r at offset r*cs: gather in place
        const ncclResult_t r = g_nccl.AllGather(buf + eb * c->rank * cs, buf, (size_t)cs,
                                                eb == 4 ? ncclFloat32 : ncclBfloat16, c->nccl_fetch, c->h2d);
        if (r != ncclSuccess) async_fail(c, SH_ERR_NCCL, "ncclAllGather(fetch): %s", g_nccl.GetErrorString(r));
      } else {  // test mode (one GPU): the other ranks' slices come over PCIe as well
        if (slo > 0) CKA(c, cudaMemcpyAsync(buf, hsrc, eb * slo, cudaMemcpyHostToDevice, c->h2d));
        if (n > shi) CKA(c, cudaMemcpyAsync(buf + eb * shi, hsrc + eb * shi, eb * (n - shi), cudaMemcpyHostToDevice, c->h2d));
      }
    }
    if (cast) CKA(c, kern::cast_bf16(stage_buf, reinterpret_cast<uint16_t*>(dst), n, c->h2d));
    CKA(c, cudaEventRecord(c->ev_arrive[y], c->h2d));
    c->h2d_bytes += slice && c->use_nccl ? eb * (shi - slo) : bytes;
    c->h2d_copies++;
    c->arrive_pub[y].store(gen);
    notify_state(c);
  });
  return SH_OK;
}

// Make sure the layer used at position p is in the ring; false if no slot can take it yet.
bool ensure_at(sh_ctx* c, int p, int cur, sh_status* st) {
  *st = SH_OK;
  const int y = c->layer_at(p);
  if (c->layer_slot[y] >= 0) return true;
  int best = -1;
  int64_t best_nu = -2;
  for (int s = 0; s < c->n_active; ++s) {
    if (c->byte_ring() && c->slot_cap[s] < c->lay[y].n_pad) continue;  // too small for this layer
    const int o = c->slot_layer[s];
    const int64_t nu = o < 0 ? kInf + 1 : next_use(c, o, cur);
    if (nu == kPinned || nu <= p) continue;
    // farthest next use (Belady); among equals (e.g. host layers done for this step) the least
    // recently used, whose gradient offload was requested first and is most likely complete
    // (fixed-byte ring: among equal next uses the smallest slot that fits -- best fit keeps the
    // large slots for the large layers)
    const bool tie_better = c->byte_ring() && best >= 0 && c->slot_cap[s] != c->slot_cap[best]
                                ? c->slot_cap[s] < c->slot_cap[best]
                                : best >= 0 && c->slot_last_use[s] < c->slot_last_use[best];
    if (nu > best_nu || (nu == best_nu && tie_better))
      best_nu = nu, best = s;
  }
  if (best < 0) return false;
  *st = issue_fetch(c, y, best, p);
  return *st == SH_OK;
}

// Common PRE work: ensure the current layer, prefetch the window ahead, wait for arrival.
sh_status pre_common(sh_ctx* c, int x, int pos) {
  sh_status st;
  const int last = std::min(pos + c->d, 2 * c->L - 1);
  for (int p = pos; p <= last; ++p) {
    const bool ok = ensure_at(c, p, pos, &st);
    if (st != SH_OK) return st;
    if (!ok) {
      if (p == pos) {
        set_error("internal: no ring slot for layer %d at position %d", x, pos);
        return SH_ERR_STATE;
      }
      break;
    }
  }
  c->slot_last_use[c->layer_slot[x]] = ++c->pos_clock;
  if (c->arrive_gen[x] > c->compute_waited[x]) {
    const int64_t gen = c->arrive_gen[x];
    if (c->arrive_by_issuer[x] &&
        !state_wait(c, [&] { return c->arrive_pub[x].load() >= gen; }, "prefetch issue"))
      return check_failed(c);
    CKC(c, cudaStreamWaitEvent(c->cs, c->ev_arrive[x], 0));
    c->compute_waited[x] = gen;
  }
  return check_failed(c);
}

void fill_param_ptrs(sh_ctx* c, int x, void** out) {
  const LayerLayout& Lx = c->lay[x];
  char* base = c->slot_param(c->layer_slot[x]);
  for (int k = 0; k < Lx.n_tensors; ++k) out[k] = base + (int64_t)c->cb * Lx.offset[k];
}

sh_status stage_g_layers(sh_ctx* c) {
  // ring reset: G layers 0..w-1 into slots 0..w-1 (compute stream), the rest empty
  for (int s = 0; s < c->n_slots; ++s) c->slot_layer[s] = -1;
  for (int x = 0; x < c->L; ++x) c->layer_slot[x] = -1;
  for (int x = 0; x < std::min(c->w, c->n_active); ++x) {  // the rest are restaged by K1 on demand
    c->slot_layer[x] = x;
    c->layer_slot[x] = x;
    char* dst = c->slot_param(x);
    if (c->bf16)
      CKC(c, kern::cast_bf16(c->g[x].master, reinterpret_cast<uint16_t*>(dst), c->lay[x].n_pad, c->cs));
    else
      CKC(c, cudaMemcpyAsync(dst, c->g[x].master, 4 * c->lay[x].n_pad, cudaMemcpyDeviceToDevice, c->cs));
  }
  return SH_OK;
}

sh_status alloc_g(sh_ctx* c, int x) {
  if (c->g[x].master) return SH_OK;
  const int64_t n = c->lay[x].n_pad;
  float* p = nullptr;
  if (cudaMalloc(&p, 3 * 4 * n) != cudaSuccess) {
    cudaGetLastError();
    set_error("cudaMalloc of GPU-optimised state for layer %d (%lld B) failed", x, (long long)(12 * n));
    return SH_ERR_OOM_DEVICE;
  }
  c->g[x].master = p;
  c->g[x].m = p + n;
  c->g[x].v = p + 2 * n;
  c->device_bytes += 12 * n;
  return SH_OK;
}

void free_g(sh_ctx* c, int x) {
  if (!c->g[x].master) return;
  cudaFree(c->g[x].master);
  c->device_bytes -= 12 * c->lay[x].n_pad;
  c->g[x] = GState{};
}

std::string shm_path(const sh_ctx* c, const char* suffix, int x = -1) {
  char b[256];
  if (x >= 0) snprintf(b, sizeof(b), "/%s.%s%d", c->shm_name.c_str(), suffix, x);
  else snprintf(b, sizeof(b), "/%s.%s", c->shm_name.c_str(), suffix);
  return b;
}

// Map (rank 0: create) a /dev/shm segment of `bytes`; page-lock it in this process.
sh_status shm_map(sh_ctx* c, const std::string& path, size_t bytes, bool create, char** out, bool touch,
                  const std::function<void(char*)>& before_touch = nullptr) {
  *out = nullptr;
  int fd = -1;
  if (create) {
    if (touch) {
      const char* mg = getenv("SH_HOST_MARGIN_GB");
      const int64_t margin = (int64_t)((mg ? atof(mg) : 3.0) * (1ll << 30));
      if ((int64_t)bytes + margin > mem_available_bytes()) {
        set_error("shared host store: %lld B requested, %lld B available", (long long)bytes,
                  (long long)mem_available_bytes());
        return SH_ERR_OOM_HOST;
      }
    }
    struct statvfs vfs;
    if (touch && statvfs("/dev/shm", &vfs) == 0 && (int64_t)vfs.f_bavail * (int64_t)vfs.f_frsize < (int64_t)bytes) {
      set_error("shared host store: /dev/shm has %lld B free, %lld B needed",
                (long long)vfs.f_bavail * (long long)vfs.f_frsize, (long long)bytes);
      return SH_ERR_OOM_HOST;
    }
    shm_unlink(path.c_str());
    fd = shm_open(path.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600);
    if (fd >= 0 && ftruncate(fd, (off_t)bytes) != 0) {
      close(fd);
      fd = -1;
    }
  } else {
    fd = shm_open(path.c_str(), O_RDWR, 0600);
  }
  if (fd < 0) {
    set_error("shm_open(%s) failed: %s", path.c_str(), strerror(errno));
    return SH_ERR_OOM_HOST;
  }
  void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (p == MAP_FAILED) {
    set_error("mmap of shared segment %s failed", path.c_str());
    return SH_ERR_OOM_HOST;
  }
  madvise(p, bytes, MADV_HUGEPAGE);
  if (create && touch && before_touch) before_touch(static_cast<char*>(p));
  if (create && touch) parallel_touch(static_cast<char*>(p), bytes, c->n_threads);
  if (touch && cudaHostRegister(p, bytes, cudaHostRegisterPortable) != cudaSuccess) {
    cudaGetLastError();
    munmap(p, bytes);
    set_error("cudaHostRegister of shared segment %s failed", path.c_str());
    return SH_ERR_OOM_HOST;
  }
  *out = static_cast<char*>(p);
  return SH_OK;
}

// Host block of layer x: [master | m | v | shadow?], 2 MiB aligned.  Shared stores map the
// segment rank 0 created (all layers are created collectively in sh_init).
// NEXT-2: a layer beyond the pinned budget lives in a file in spill_dir -- the paper's swap file on the
// secondary storage -- read and written with O_DIRECT bulk requests (io_uring), so
// the tier's RAM is bounded by its pinned staging / bounce buffers instead of the page cache.  The file
// is unlinked right away (nothing is left behind on a crash); space is reserved with posix_fallocate so
// a full disk fails here, not in the middle of a step.  File systems without O_DIRECT (tmpfs) get a
// plain descriptor and the same aligned transfers.
sh_status spill_block_alloc(sh_ctx* c, int x, size_t bytes, int* fd_out) {
  *fd_out = -1;
  char path[4096];
  snprintf(path, sizeof(path), "%s/sh_spill_%d_%p_%d.bin", c->spill_dir.c_str(), (int)getpid(), (void*)c, x);
  int fd = open(path, O_RDWR | O_CREAT | O_EXCL | O_DIRECT, 0600);
  bool direct = fd >= 0;
  if (fd < 0 && errno == EINVAL) fd = open(path, O_RDWR | O_CREAT | O_EXCL, 0600);
  if (fd < 0) {
    set_error("spill tier: open(%s): %s", path, strerror(errno));
    return SH_ERR_OOM_HOST;
  }
  unlink(path);
  const int e = posix_fallocate(fd, 0, (off_t)bytes);
  if (e != 0) {
    close(fd);
    set_error("spill tier: posix_fallocate of %lld B in %s: %s", (long long)bytes, c->spill_dir.c_str(), strerror(e));
    return SH_ERR_OOM_HOST;
  }
  if (c->n_spilled == 0) c->spill_direct = direct;
  else c->spill_direct = c->spill_direct && direct;
  *fd_out = fd;
  return SH_OK;
}

// Pinned buffers of the tier, allocated with the first spilled layer: two bounce buffers for fetches
// and SH_SPILL_STAGING (default 3) staging copies for the CPU updates, plus its two I/O threads.
sh_status ensure_bounce(sh_ctx* c) {
  if (c->bounce[0]) return SH_OK;
  const size_t b = align_up(4 * c->max_pad, 1 << 21);  // fp32 fetch is the largest
  for (int k = 0; k < 2; ++k) {
    sh_status st = host_block_alloc(b, c->n_threads, &c->bounce[k], c->land_node, &c->numa_bound);
    if (st != SH_OK) return st;
    CKC(c, cudaEventCreateWithFlags(&c->ev_bounce[k], cudaEventDisableTiming));
    CKC(c, cudaEventRecord(c->ev_bounce[k], c->h2d));
    c->host_bytes += b;
  }
  c->bounce_bytes = b;
  const char* e = getenv("SH_SPILL_STAGING");
  const int n_stg = std::max(1, e ? atoi(e) : 3);
  int64_t fb = 0;
  for (int x = 0; x < c->L; ++x) fb = std::max(fb, sp_file_bytes(c, x));
  c->stg_bytes = align_up(fb, 1 << 21);
  for (int k = 0; k < n_stg; ++k) {
    char* p = nullptr;
    sh_status st = host_block_alloc(c->stg_bytes, c->n_threads, &p, c->land_node, &c->numa_bound);
    if (st != SH_OK) return st;
    c->stg_all.push_back(p);
    c->stg_free.push_back(p);
    c->host_bytes += c->stg_bytes;
  }
  if (!c->spill_threads) {
    c->spill_rd.start();
    c->spill_wr.start();
    c->spill_threads = true;
  }
  return SH_OK;
}

// Split master (R25) on n elements in parallel: fp32 -> (hi, lo) planes, and back.
void split_par(sh_ctx* c, const float* src, uint16_t* hi, uint16_t* lo, int64_t b, int64_t e) {
  const int nt = std::max(1, std::min(c->n_threads, 16));
  const int64_t chunk = align_up((e - b + nt - 1) / nt, 16);
  std::vector<std::thread> ts;
  for (int64_t x0 = b; x0 < e; x0 += chunk)
    ts.emplace_back([=] { cpu::split_range(src, hi, lo, x0, std::min(e, x0 + chunk)); });
  for (auto& t : ts) t.join();
}
void join_par(sh_ctx* c, const uint16_t* hi, const uint16_t* lo, float* dst, int64_t b, int64_t e) {
  const int nt = std::max(1, std::min(c->n_threads, 16));
  const int64_t chunk = align_up((e - b + nt - 1) / nt, 16);
  std::vector<std::thread> ts;
  for (int64_t x0 = b; x0 < e; x0 += chunk)
    ts.emplace_back([=] { cpu::join_range(hi, lo, dst, x0, std::min(e, x0 + chunk)); });
  for (auto& t : ts) t.join();
}

// A kAlign-aligned temporary host buffer (registration, window changes and reads of spilled layers).
struct AlignedBuf {
  void* p = nullptr;
  explicit AlignedBuf(size_t bytes) {
    if (posix_memalign(&p, spill::kAlign, align_up((int64_t)bytes, (int64_t)spill::kAlign)) != 0) p = nullptr;
  }
  ~AlignedBuf() { free(p); }
  float* f() const { return static_cast<float*>(p); }
  char* b() const { return static_cast<char*>(p); }
};

void release_host_layer(sh_ctx* c, int x) {
  auto& hb = c->hblocks[x];
  if (!hb.p && hb.fd < 0) return;
  if (hb.fd >= 0) {
    close(hb.fd);
    c->spill_bytes -= hb.bytes;
    c->n_spilled--;
    c->spilled[x] = 0;
  } else {
    host_block_free(hb.p, hb.bytes);
    c->host_bytes -= hb.bytes;
  }
  hb = {};
  c->h_master[x] = c->h_m[x] = c->h_v[x] = nullptr;
  c->h_shadow[x] = nullptr;
  c->h_lo[x] = nullptr;
  auto& sb = c->hshadow[x];
  if (sb.p) {
    host_block_free(sb.p, sb.bytes);
    c->host_bytes -= sb.bytes;
    sb = {};
  }
}

// SH_FLAG_LATE_SHADOW: give every host-optimised layer without one a bf16 shadow in its own pinned
// block (the host RAM the GPU set gave back), written from the master with the CPU Adam's RNE cast,
// so its prefetches move 2 instead of 4 B/param over the link.  Stops quietly at the first block
// the RAM refuses (those layers keep the fp32 fetch + K1 cast).  Between steps, engine idle.
sh_status enable_late_shadow(sh_ctx* c) {
  if (!c->bf16 || c->shared) return SH_OK;
  for (int x = c->w; x < c->L; ++x) {
    if (c->h_shadow[x] || !c->h_master[x]) continue;
    const int64_t n = c->lay[x].n_pad;
    const size_t bytes = align_up(2 * n, 1 << 21);
    char* p = nullptr;
    if (host_block_alloc(bytes, c->n_threads, &p, c->layer_node[x], &c->numa_bound) != SH_OK) {
      clear_error();
      break;
    }
    c->hshadow[x] = {p, bytes, -1};
    c->host_bytes += bytes;
    uint16_t* sh16 = reinterpret_cast<uint16_t*>(p);
    const int nt = std::max(1, c->n_threads);
    std::vector<std::thread> ts;
    const int64_t chunk = align_up((n + nt - 1) / nt, 16);
    for (int t = 0; t < nt; ++t) {
      const int64_t b = t * chunk, e = std::min(n, b + chunk);
      if (b < e) ts.emplace_back([=] { cpu::cast_bf16_range(c->h_master[x], sh16, b, e); });
    }
    for (auto& th : ts) th.join();
    c->h_shadow[x] = sh16;
  }
  return SH_OK;
}

sh_status ensure_host_layer(sh_ctx* c, int x) {
  if (c->hblocks[x].p || c->hblocks[x].fd >= 0) return SH_OK;
  const int64_t n = c->lay[x].n_pad;
  size_t bytes = align_up(12 * n + (c->shadow ? 2 * n : 0), 1 << 21);  // split: [hi | lo | m | v], 12 B
  char* p = nullptr;
  int fd = -1;
  sh_status st = SH_OK;
  if (c->shared) {
    // data parallel: rank r's slice of each of the four arrays on GPU r's node
    auto place = [c, x, n](char* base) {
      if (c->slice_node.empty()) return;
      const int64_t cs = align_up((n + c->W - 1) / c->W, kPad);
      const int n_arr = c->split ? 4 : c->shadow ? 4 : 3;
      for (int r = 0; r < c->W; ++r) {
        const int64_t lo = std::min(n, (int64_t)r * cs), hi = std::min(n, (int64_t)(r + 1) * cs);
        if (lo >= hi || c->slice_node[r] == numa::kNone) continue;
        for (int a = 0; a < n_arr; ++a) {
          // arrays: master, m, v[, shadow]  or (split) hi, lo, m, v
          const int64_t esz = c->split ? (a < 2 ? 2 : 4) : (a < 3 ? 4 : 2);
          const int64_t off = c->split ? (a < 2 ? 2 * a * n : 4 * (a - 1) * n) : (a < 3 ? 4 * a * n : 12 * n);
          if (numa::bind_range(base + off + esz * lo, (size_t)(esz * (hi - lo)), c->slice_node[r]))
            c->numa_bound.fetch_add(esz * (hi - lo));
        }
      }
    };
    st = shm_map(c, shm_path(c, "L", x), bytes, c->rank == 0, &p, true, place);
  } else {
    const bool can_spill = !c->spill_dir.empty();
    bool spill = can_spill && c->pin_budget > 0 && (int64_t)(c->host_bytes + bytes) > c->pin_budget;
    if (!spill) {
      st = host_block_alloc(bytes, c->n_threads, &p, c->layer_node[x], &c->numa_bound);
      if (st == SH_ERR_OOM_HOST && can_spill) {  // host RAM exhausted: overflow to the spill tier
        clear_error();
        spill = true;
      }
    }
    if (spill) {
      bytes = (size_t)sp_file_bytes(c, x);
      st = ensure_bounce(c);
      if (st == SH_OK) st = spill_block_alloc(c, x, bytes, &fd);
    }
  }
  if (st != SH_OK) return st;
  c->hblocks[x] = {p, bytes, fd};
  if (fd >= 0) {  // no host mapping: h_master / m / v / shadow stay null
    c->spilled[x] = 1;
    c->spill_bytes += bytes;
    c->n_spilled++;
    return SH_OK;
  }
  c->host_bytes += bytes;
  float* b = reinterpret_cast<float*>(p);
  if (c->split) {
    c->h_shadow[x] = reinterpret_cast<uint16_t*>(p);
    c->h_lo[x] = reinterpret_cast<uint16_t*>(p) + n;
    c->h_m[x] = b + n;
    c->h_v[x] = b + 2 * n;
    return SH_OK;
  }
  c->h_master[x] = b;
  c->h_m[x] = b + n;
  c->h_v[x] = b + 2 * n;
  if (c->shadow) c->h_shadow[x] = reinterpret_cast<uint16_t*>(b + 3 * n);
  return SH_OK;
}

sh_status ensure_gbufs(sh_ctx* c, int w) {
  if (!c->k2_layer || (w <= 0 && c->cfg.window == 0)) return SH_OK;
  // allocated up front (the window solver sees them as used).  Single GPU: the per-layer K2 runs
  // on the compute stream, in order, so two buffers never wait; data parallel: K2 runs on the comm
  // stream behind the all-reduce, four keep BP from waiting on it
  int want = c->dp ? 4 : 2;
  if (c->cfg.flags & SH_FLAG_KEEP_GRADS) want = std::max(want, w);  // one per GPU-optimised layer
  while ((int)c->gbuf.size() < want) {
    float* p = nullptr;
    if (cudaMalloc(&p, 4 * c->max_pad) != cudaSuccess) {
      cudaGetLastError();
      set_error("cudaMalloc of a GPU-optimised-layer grad buffer (%lld B) failed", (long long)(4 * c->max_pad));
      return SH_ERR_OOM_DEVICE;
    }
    cudaEvent_t a = nullptr, b = nullptr;
    if (cudaEventCreateWithFlags(&a, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&b, cudaEventDisableTiming) != cudaSuccess) {
      set_error("cudaEventCreate failed");
      return SH_ERR_CUDA;
    }
    cudaEventRecord(a, c->cs);
    c->gbuf.push_back(p);
    c->ev_gbuf_free.push_back(a);
    c->ev_gbuf_ready.push_back(b);
    c->gbuf_owner.push_back(-1);
    c->device_bytes += 4 * c->max_pad;
  }
  return SH_OK;
}

// Grow-only ring.  Called with the engine idle: every slot's content can be
// re-derived (GPU-optimised layers from their HBM masters, host layers from the host store), so
// the old ring is released BEFORE the new one is allocated (never both at once).  On failure the
// ring is left unallocated and the caller retries with fewer slots.
// shrink (a decoupled ring, engine idle): allocate exactly n_slots even if fewer than now -- the HBM
// goes to the GPU-optimised set the solver sized next to it (R27); bookkeeping vectors keep their size.
sh_status alloc_ring(sh_ctx* c, int n_slots, bool shrink = false) {
  if (c->ring && (n_slots == c->n_slots || (n_slots < c->n_slots && !shrink))) return SH_OK;
  if (c->ring) {
    cudaDeviceSynchronize();
    cudaFree(c->ring);
    c->device_bytes -= c->ring_bytes_for(c->ring_alloc);
    c->ring = nullptr;
    c->ring_alloc = 0;
  }
  if (!shrink) n_slots = std::max(n_slots, c->n_slots);
  char* r = nullptr;
  if (cudaMalloc(&r, c->ring_bytes_for(n_slots)) != cudaSuccess) {
    cudaGetLastError();
    // put the previous ring back (it fitted before) so the context stays usable
    if (c->n_slots > 0 && cudaMalloc(&r, c->ring_bytes_for(c->n_slots)) == cudaSuccess) {
      c->ring = r;
      c->ring_alloc = c->n_slots;
      c->device_bytes += c->ring_bytes_for(c->n_slots);
    } else {
      cudaGetLastError();
      async_fail(c, SH_ERR_OOM_DEVICE, "ring re-allocation failed");
    }
    set_error("cudaMalloc of %d ring slots (%lld B each) failed", n_slots, (long long)c->slot_bytes);
    return SH_ERR_OOM_DEVICE;
  }
  c->ring = r;
  c->ring_alloc = n_slots;
  c->device_bytes += c->ring_bytes_for(n_slots);
  cudaMemset(r, 0, c->ring_bytes_for(n_slots));
  const int cap = std::max((int)c->slot_layer.size(), n_slots);  // bookkeeping vectors never shrink
  const int old_cap = (int)c->slot_layer.size();
  c->slot_layer.assign(cap, -1);  // (a re-allocated ring holds nothing)
  c->slot_last_use.resize(cap, 0);
  c->ev_param_free.resize(cap, nullptr);
  c->ev_grad_done.resize(cap, nullptr);
  c->ev_grad_free.resize(cap, nullptr);
  c->ev_reduced.resize(cap, nullptr);
  c->ev_k3_buf.resize(cap, nullptr);
  c->gradfree_gen.resize(cap, 0);
  c->gradfree_waited.resize(cap, 0);
  c->gb_owner.assign(cap, -1);  // (engine idle: every pool buffer is free)
  c->gb_free_seq.assign(cap, 0);
  auto pub = std::make_unique<std::atomic<int64_t>[]>(cap);
  for (int s = 0; s < cap; ++s) pub[s].store(s < old_cap ? c->gradfree_pub[s].load() : 0);
  c->gradfree_pub = std::move(pub);
  for (int s = 0; s < cap; ++s) {
    if (c->ev_param_free[s]) continue;
    for (auto* v : {&c->ev_param_free, &c->ev_grad_done, &c->ev_grad_free, &c->ev_reduced, &c->ev_k3_buf})
      if (cudaEventCreateWithFlags(&(*v)[s], cudaEventDisableTiming) != cudaSuccess) {
        set_error("cudaEventCreate failed");
        return SH_ERR_CUDA;
      }
    // a fresh slot is free: record once so every wait has a completed event
    cudaEventRecord(c->ev_param_free[s], c->cs);
    cudaEventRecord(c->ev_grad_free[s], c->cs);
  }
  c->n_slots = n_slots;
  return SH_OK;
}

sh_status sync_all(sh_ctx* c) {
  c->ih2d.drain();
  c->id2h.drain();
  for (cudaStream_t s : {c->cs, c->h2d, c->d2h, c->stage, c->comm, c->k3s, c->hyb_in, c->hyb_k, c->hyb_out})
    if (s) {
      sh_status st = stream_sync(c, s);
      if (st != SH_OK) return st;
    }
  // all host layers updated for the steps taken so far
  if (!state_wait(c, [&] {
        for (int x = 0; x < c->L; ++x)
          if (!c->is_g(x) && !ready_at_least(c, x, c->step)) return false;
        return true;
      }, "CPU Adam drain"))
    return check_failed(c);
  for (auto& P : c->prof) prof_harvest(c, P);
  return check_failed(c);
}

// Forget every ring mapping: each layer is fetched / K1-restaged again at its next use (always
// valid between steps: GPU-optimised layers restage from their HBM masters, host layers fetch).
void clear_ring_map(sh_ctx* c) {
  for (int s = 0; s < (int)c->slot_layer.size(); ++s) c->slot_layer[s] = -1;
  for (int x = 0; x < c->L; ++x) c->layer_slot[x] = -1;
}

// Move the G boundary from c->w to w_new (between steps, everything idle).
sh_status apply_window(sh_ctx* c, int w_new) {
  sh_status st = sync_all(c);
  if (st != SH_OK) return st;
  const int w_old = c->w;
  // leaving G: HBM -> host store (bitwise), shadow recomputed with the same RNE
  for (int x = w_new; x < w_old; ++x) {
    st = ensure_host_layer(c, x);
    if (st != SH_OK) return st;
    if (c->spilled[x]) {  // NEXT-2: into the layer's spill file
      const int64_t n = c->lay[x].n_pad, rb = sp_rb(c, x), fb = sp_file_bytes(c, x);
      AlignedBuf t(fb);
      if (!t.p) {
        set_error("apply_window: no memory for a %lld B spill staging copy", (long long)fb);
        return SH_ERR_OOM_HOST;
      }
      std::memset(t.p, 0, fb);
      if (c->split) {  // region 0 = [hi | lo]
        std::vector<float> mst(n);
        CKC(c, cudaMemcpy(mst.data(), c->g[x].master, 4 * n, cudaMemcpyDeviceToHost));
        uint16_t* h16 = reinterpret_cast<uint16_t*>(t.b());
        split_par(c, mst.data(), h16, h16 + n, 0, n);
      } else {
        CKC(c, cudaMemcpy(t.b(), c->g[x].master, 4 * n, cudaMemcpyDeviceToHost));
      }
      CKC(c, cudaMemcpy(t.b() + rb, c->g[x].m, 4 * n, cudaMemcpyDeviceToHost));
      CKC(c, cudaMemcpy(t.b() + 2 * rb, c->g[x].v, 4 * n, cudaMemcpyDeviceToHost));
      if (c->shadow) cpu::cast_bf16_range(t.f(), reinterpret_cast<uint16_t*>(t.b() + 3 * rb), 0, n);
      st = spill_file_io(c, true, x, t.p, fb);
      if (st != SH_OK) return st;
      c->ready[x].store(c->step);
      free_g(c, x);
      continue;
    }
    // every rank holds the same GPU state; each writes its own slice of the (shared) store
    const int64_t lo = c->slo[x], nb = 4 * (c->shi[x] - c->slo[x]);
    if (c->split) {
      std::vector<float> mst(c->shi[x] - lo);
      CKC(c, cudaMemcpy(mst.data(), c->g[x].master + lo, nb, cudaMemcpyDeviceToHost));
      split_par(c, mst.data() - lo, c->h_shadow[x], c->h_lo[x], lo, c->shi[x]);
    } else {
      CKC(c, cudaMemcpy(c->h_master[x] + lo, c->g[x].master + lo, nb, cudaMemcpyDeviceToHost));
    }
    CKC(c, cudaMemcpy(c->h_m[x] + lo, c->g[x].m + lo, nb, cudaMemcpyDeviceToHost));
    CKC(c, cudaMemcpy(c->h_v[x] + lo, c->g[x].v + lo, nb, cudaMemcpyDeviceToHost));
    if (c->h_shadow[x] && !c->split) cpu::cast_bf16_range(c->h_master[x], c->h_shadow[x], lo, c->shi[x]);
    c->ready[x].store(c->step);
    free_g(c, x);
  }
  if (w_new < w_old && c->shared) {
    if (!shm_barrier(c, 2, "window change (slices written)")) return check_failed(c);
    if (c->rank == 0)
      for (int x = w_new; x < w_old; ++x) {
        c->ctl->cnt[x].store((int64_t)c->W * c->step);
        c->ctl->cnt[c->L + x].store((int64_t)c->W * c->step);
      }
    if (!shm_barrier(c, 3, "window change (counters)")) return check_failed(c);
  }
  // ring first (the old one is released inside), then the joining layers' HBM states (rolled
  // back on failure so the caller can retry with a smaller window)
  st = alloc_ring(c, c->ring_for(w_new), c->ring_cap > 0 && !c->byte_ring());
  if (st != SH_OK) {
    clear_ring_map(c);  // a re-allocated ring holds no valid copy
    return st;
  }
  for (int x = w_old; x < w_new; ++x) {
    st = alloc_g(c, x);
    if (st != SH_OK) {
      for (int y = w_old; y < w_new; ++y) free_g(c, y);
      clear_ring_map(c);
      return st;
    }
    const int64_t n = c->lay[x].n_pad;
    if (c->spilled[x]) {  // NEXT-2: from the layer's spill file
      const int64_t rb = sp_rb(c, x);
      AlignedBuf t(3 * rb);
      if (!t.p) {
        set_error("apply_window: no memory for a spill staging copy");
        return SH_ERR_OOM_HOST;
      }
      st = spill_file_io(c, false, x, t.p, 3 * rb);
      if (st != SH_OK) return st;
      if (c->split) {
        std::vector<float> mst(n);
        const uint16_t* h16 = reinterpret_cast<const uint16_t*>(t.b());
        join_par(c, h16, h16 + n, mst.data(), 0, n);
        CKC(c, cudaMemcpy(c->g[x].master, mst.data(), 4 * n, cudaMemcpyHostToDevice));
      } else {
        CKC(c, cudaMemcpy(c->g[x].master, t.b(), 4 * n, cudaMemcpyHostToDevice));
      }
      CKC(c, cudaMemcpy(c->g[x].m, t.b() + rb, 4 * n, cudaMemcpyHostToDevice));
      CKC(c, cudaMemcpy(c->g[x].v, t.b() + 2 * rb, 4 * n, cudaMemcpyHostToDevice));
      continue;
    }
    if (c->split) {
      std::vector<float> mst(n);
      join_par(c, c->h_shadow[x], c->h_lo[x], mst.data(), 0, n);
      CKC(c, cudaMemcpy(c->g[x].master, mst.data(), 4 * n, cudaMemcpyHostToDevice));
    } else {
      CKC(c, cudaMemcpy(c->g[x].master, c->h_master[x], 4 * n, cudaMemcpyHostToDevice));
    }
    CKC(c, cudaMemcpy(c->g[x].m, c->h_m[x], 4 * n, cudaMemcpyHostToDevice));
    CKC(c, cudaMemcpy(c->g[x].v, c->h_v[x], 4 * n, cudaMemcpyHostToDevice));
  }
  st = ensure_gbufs(c, w_new);
  if (st != SH_OK) {
    for (int y = w_old; y < w_new; ++y) free_g(c, y);
    clear_ring_map(c);
    return st;
  }
  c->w = w_new;
  c->n_active = c->ring_for(w_new);
  c->d = c->n_active - 1;
  st = stage_g_layers(c);
  if (st != SH_OK) return st;
  CKC(c, cudaStreamSynchronize(c->cs));
  // the joining layers' masters / m / v now live in HBM: give their host blocks back (a private
  // store re-allocates one if the layer leaves the GPU set again; shared segments stay mapped)
  if (!c->shared)
    for (int x = w_old; x < w_new; ++x) release_host_layer(c, x);
  return SH_OK;
}

// Grow the host landing ring to D_new buffers (private store, between steps): a fresh pinned block,
// the two clip-coefficient words carried over, every buffer's use counter restarted.  Lets the
// autotuner decouple the ring from the GPU-optimised set (R22) once the layers joining that set
// have given their host blocks back.
sh_status grow_landing(sh_ctx* c, int D_new) {
  if (D_new <= c->D || c->shared) return SH_OK;
  sh_status st = sync_all(c);
  if (st != SH_OK) return st;
  const int64_t lb = align_up(4 * c->max_pad, 4096);
  const size_t bytes = align_up((int64_t)D_new * lb + 4096, 1 << 21);
  char* p = nullptr;
  st = host_block_alloc(bytes, c->n_threads, &p, c->land_node, &c->numa_bound);
  if (st != SH_OK) return st;
  const float coef0 = c->h_coef[0], coef1 = c->h_coef[1];
  host_block_free(c->hland.p, c->hland.bytes);
  c->host_bytes -= c->hland.bytes;
  c->hland = {p, bytes};
  c->host_bytes += bytes;
  c->D = D_new;
  c->landing.resize(D_new);
  for (int k = 0; k < D_new; ++k) c->landing[k] = reinterpret_cast<float*>(p + (int64_t)k * lb);
  c->h_coef = reinterpret_cast<float*>(p + (int64_t)D_new * lb);
  c->h_coef[0] = coef0;
  c->h_coef[1] = coef1;
  {
    std::lock_guard<std::mutex> g(c->smu);
    c->land_free.clear();
    for (int k = 0; k < D_new; ++k) c->land_free.push_back(k);
  }
  c->landing_owner.assign(D_new, -1);
  c->last_landing.assign(c->L, -1);
  return SH_OK;
}

// K4 on the compute stream: dst = (dst + Σ_e src[e]) / K in a fixed order (NEXT-3).
sh_status exec_fold(sh_ctx* c, float* dst, const std::vector<float*>& src, int64_t n) {
  kern::K4Args a{};
  a.dst = dst;
  a.n_src = (int)src.size();
  for (int e = 0; e < a.n_src; ++e) a.src[e] = src[e];
  a.n = n;
  a.inv_k = (float)(1.0 / (double)c->K);
  CKC(c, kern::exec_reduce(a, c->cs));
  return SH_OK;
}

sh_status push_k2(sh_ctx* c, kern::K2Args& a, int64_t* bytes, int* launches) {
  if (a.n_entries == 0) return SH_OK;
  for (int i = 0; i < a.n_entries; ++i) *bytes += (c->bf16 ? 30 : 32) * a.e[i].n;
  a.sched = c->k2_sched_cs;
  CKC(c, kern::adamw_multi(a, c->cs));
  (*launches)++;
  a.n_entries = 0;
  return SH_OK;
}

sh_status nccl_check(sh_ctx* c, ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return SH_OK;
  async_fail(c, SH_ERR_NCCL, "%s: %s", what, g_nccl.GetErrorString(r));
  set_error("%s: %s", what, g_nccl.GetErrorString(r));
  return SH_ERR_NCCL;
}

// ---- collectives of the data-parallel path.  NCCL over NVLink in production.
// SH_FLAG_TEST_HOST_COLLECTIVE runs the same three operations through the shared host segment on the
// driver thread -- every rank sums the ranks' contributions in rank order, so the results are
// bitwise identical on all ranks -- which lets several ranks with DIFFERENT data share one GPU and
// checks the averaging itself against the oracle's global-batch mean (reading R13).
enum CollOp { kAllReduceAvg, kReduceScatterAvg, kAllGatherF64 };

sh_status coll_host(sh_ctx* c, CollOp op, void* buf, int64_t n, int64_t lo, int64_t hi, void* out, cudaStream_t st) {
  const int64_t eb = op == kAllGatherF64 ? 8 : 4;
  if (n * eb > c->hc_count * 4) {
    set_error("host collective: %lld elements exceed the segment", (long long)n);
    return SH_ERR_INVALID;
  }
  float* mine = c->hc_seg + (int64_t)c->rank * c->hc_count;
  CKC(c, cudaMemcpyAsync(mine, buf, n * eb, cudaMemcpyDeviceToHost, st));
  CKC(c, cudaStreamSynchronize(st));
  const int64_t k = ++c->hc_seq;
  c->ctl->hc_arrive[c->rank].store(k, std::memory_order_release);
  auto all_at = [&](std::atomic<int64_t>* a) {
    for (int r = 0; r < c->W; ++r)
      if (a[r].load(std::memory_order_acquire) < k) return false;
    return true;
  };
  if (!state_wait(c, [&] { return all_at(c->ctl->hc_arrive); }, "host collective (contributions)"))
    return check_failed(c);
  void* dst;
  const void* src;
  int64_t bytes;
  if (op == kAllGatherF64) {
    for (int r = 0; r < c->W; ++r)
      std::memcpy(reinterpret_cast<char*>(c->hc_tmp) + (int64_t)r * n * 8, c->hc_seg + (int64_t)r * c->hc_count, n * 8);
    dst = out;
    src = c->hc_tmp;
    bytes = (int64_t)c->W * n * 8;
  } else {
    const int64_t b = op == kReduceScatterAvg ? lo : 0, e = op == kReduceScatterAvg ? hi : n;
    const float inv = (float)(1.0 / (double)c->W);
    for (int64_t i = b; i < e; ++i) {
      float acc = c->hc_seg[i];
      for (int r = 1; r < c->W; ++r) acc = acc + c->hc_seg[(int64_t)r * c->hc_count + i];
      c->hc_tmp[i] = acc * inv;
    }
    dst = static_cast<float*>(buf) + b;
    src = c->hc_tmp + b;
    bytes = 4 * (e - b);
  }
  c->ctl->hc_done[c->rank].store(k, std::memory_order_release);
  if (bytes > 0) {
    CKC(c, cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, st));
    CKC(c, cudaStreamSynchronize(st));  // hc_tmp is reused by the next call
  }
  // nobody rewrites its contribution before every rank has read this round's
  if (!state_wait(c, [&] { return all_at(c->ctl->hc_done); }, "host collective (completion)"))
    return check_failed(c);
  return SH_OK;
}

// Average of a gradient buffer over the ranks (every rank gets all n elements).
sh_status coll_allreduce_avg(sh_ctx* c, float* buf, int64_t n, cudaStream_t st, const char* what) {
  if (c->host_coll) return coll_host(c, kAllReduceAvg, buf, n, 0, n, nullptr, st);
  if (!c->use_nccl) return SH_OK;  // SH_FLAG_TEST_NO_COLLECTIVE: identical data, the average is the identity
  return nccl_check(c, g_nccl.AllReduce(buf, buf, n, ncclFloat, ncclAvg, c->nccl, st), what);
}

// Host layer x with a shared store: rank r offloads and CPU-updates only its slice [slo, shi), so it
// needs only that slice of the average -- a reduce-scatter (half the NVLink bytes of an all-reduce,
// NEXT-1).  In place: slice r of the W*cs-element buffer receives the result (NCCL's in-place form).
sh_status coll_reduce_scatter_avg(sh_ctx* c, float* buf, int x, cudaStream_t st) {
  const int64_t n = c->lay[x].n_pad, cs = align_up((n + c->W - 1) / c->W, kPad);
  if (c->host_coll) return coll_host(c, kReduceScatterAvg, buf, n, c->slo[x], c->shi[x], nullptr, st);
  if (!c->use_nccl) return SH_OK;
  return nccl_check(c, g_nccl.ReduceScatter(buf, buf + (int64_t)c->rank * cs, (size_t)cs, ncclFloat, ncclAvg,
                                            c->nccl, st),
                    "ncclReduceScatter(layer grads)");
}

// Reduce-scattered host layers leave each rank with the sum of squares of its slice only: gather the
// per-rank partials and fold them in rank order (identical on every rank) before the norm.
sh_status coll_fold_partials(sh_ctx* c, cudaStream_t st) {
  if (!c->rs_host) return SH_OK;
  const int n = c->L + 1;
  sh_status r = SH_OK;
  if (c->host_coll)
    r = coll_host(c, kAllGatherF64, c->partials, n, 0, n, c->partials_all, st);
  else
    r = nccl_check(c, g_nccl.AllGather(c->partials, c->partials_all, (size_t)n, ncclFloat64, c->nccl, st),
                   "ncclAllGather(norm partials)");
  if (r != SH_OK) return r;
  CKC(c, kern::fold_partials(c->partials_all, c->W, n, c->w, c->partials, st));
  return SH_OK;
}

// ---- gradient pool + offload scheduler.  Without enough host landing buffers the CPU
// Adam paces the offloads; a FIFO offload queue then leaves the LOWEST layers' gradients (produced
// last in BP) waiting in HBM behind the high ones at the end of BP, so the next FP -- which needs the
// lowest layer first -- waits for the whole backlog (measured: 0.78 s of a 3.76 s c4max step).  The
// scheduler offloads the lowest pending layer whenever a landing buffer is free, so the layers the
// next FP needs first are updated first and the high layers' updates overlap that FP.  Gradients
// wait in the pool (the ring's grad halves, any buffer for any layer), not in the slot their
// layer's parameters happened to occupy, so the out-of-order offloads never block BP.

// A free pool buffer of at least n elements for layer x (blocks until one's offload is issued).
int take_grad_buffer(sh_ctx* c, int x, int64_t n) {
  // among the free buffers (offload issued) prefer one whose offload has already COMPLETED, then the
  // one released longest ago: taking the buffer of the offload issued last would make the compute
  // stream wait for that copy (~17 ms for an h4096 layer)
  int b = -1;
  auto pick = [&] {
    b = -1;
    bool b_done = false;
    for (int k = 0; k < c->n_slots; ++k) {
      if (c->gb_owner[k] != -1 || c->gradfree_pub[k].load() < c->gradfree_gen[k]) continue;
      if (c->byte_ring() && c->slot_cap[k] < n) continue;
      const bool done = cudaEventQuery(c->ev_grad_free[k]) == cudaSuccess;
      if (!done) cudaGetLastError();  // (cudaErrorNotReady is not sticky; clear it anyway)
      bool better;
      if (b < 0) better = true;
      else if (c->byte_ring() && c->slot_cap[k] != c->slot_cap[b]) better = c->slot_cap[k] < c->slot_cap[b];  // best fit
      else if (done != b_done) better = done;
      else better = c->gb_free_seq[k] < c->gb_free_seq[b];
      if (better) b = k, b_done = done;
    }
    return b >= 0;
  };
  {
    std::unique_lock<std::mutex> g(c->smu);
    if (pick()) {
      c->gb_owner[b] = x;
      return b;
    }
  }
  c->grad_starved.store(1);
  const bool got = state_wait(c, pick, "a free gradient buffer");
  c->grad_starved.store(0);
  if (c->cpu_throttle > 0) c->pcv.notify_all();
  if (!got) return -1;
  std::lock_guard<std::mutex> g(c->smu);
  if (!pick()) return -1;  // (failed meanwhile)
  c->gb_owner[b] = x;
  return b;
}

void release_grad_buffer(sh_ctx* c, int b) {
  {
    std::lock_guard<std::mutex> g(c->smu);
    c->gb_owner[b] = -1;
    c->gb_free_seq[b] = ++c->gb_free_ctr;
  }
  c->scv.notify_all();
}

// ---------------------------------------------------------------------------- R28 hybrid update
struct HybDone {
  sh_ctx* c;
  int layer;
  int64_t step;
};

void CUDART_CB hyb_done_cb(void* arg) {  // CUDA driver thread: no CUDA calls
  std::unique_ptr<HybDone> h(static_cast<HybDone*>(arg));
  mark_updated(h->c, h->layer, h->step);  // host hi / lo / m / v written back: fetchable again
}

// At BP PRE(y): issue the staging fetch (host lo / m / v -> HBM) of every hybrid layer among the next
// D = S - 1 backward positions (y, y-1, ..., y-D) not yet issued this step, into the staging buffers
// round-robin.  A buffer's previous user is the hybrid layer S fetches back, whose K2S and write-back
// were enqueued at its POST (it is above y - D); the copy waits for that write-back on the GPU.
sh_status hyb_issue(sh_ctx* c, int y) {
  const int S = (int)c->hyb_stg.size();
  for (int x = y; x >= std::max(c->w, y - (S - 1)); --x) {
    if (!c->is_hyb(x) || c->hyb_issued[x] == c->step) continue;
    // the host planes are current once the layer's previous update (CPU or write-back) has landed
    if (!state_wait(c, [&] { return ready_at_least(c, x, c->step); }, "host update before a hybrid fetch"))
      return check_failed(c);
    const int i = (int)(c->hyb_rr++ % S);
    const int64_t n = c->lay[x].n_pad;
    CKC(c, cudaStreamWaitEvent(c->hyb_in, c->ev_stg_free[i], 0));
    CKC(c, cudaMemcpyAsync(c->hyb_stg[i], c->h_lo[x], 10 * n, cudaMemcpyHostToDevice, c->hyb_in));  // [lo | m | v]
    CKC(c, cudaEventRecord(c->ev_stg_in[i], c->hyb_in));
    c->hyb_stg_of[x] = i;
    c->hyb_issued[x] = c->step;
    c->h2d_bytes += 10 * n;
    c->hyb_h2d += 10 * n;
    c->h2d_copies++;
  }
  return SH_OK;
}

// At BP POST(x) of a hybrid layer (its K3 already on the compute stream): K2S on the split master --
// hi = the compute copy in ring slot s (updated in place), lo / m / v in the staging buffer, grads in
// pool buffer gb -- then the write-back of hi / lo / m / v to the host block; the layer counts as
// updated (ready) when the write-back lands, and the next FP of x uses the updated slot copy.
sh_status hyb_update(sh_ctx* c, int x, int s, int gb) {
  const int i = c->hyb_stg_of[x];
  if (i < 0 || c->hyb_issued[x] != c->step) {
    set_error("internal: hybrid layer %d has no staging fetch for step %lld", x, (long long)c->step);
    return SH_ERR_STATE;
  }
  const int64_t n = c->lay[x].n_pad;
  char* stg = c->hyb_stg[i];
  CKC(c, cudaEventRecord(c->ev_grad_done[gb], c->cs));
  CKC(c, cudaStreamWaitEvent(c->hyb_k, c->ev_grad_done[gb], 0));
  CKC(c, cudaStreamWaitEvent(c->hyb_k, c->ev_stg_in[i], 0));
  kern::K2SplitArgs a{};
  a.sc = c->sc;
  a.hi = reinterpret_cast<uint16_t*>(c->slot_param(s));
  a.lo = reinterpret_cast<uint16_t*>(stg);
  a.m = reinterpret_cast<float*>(stg + 2 * n);
  a.v = reinterpret_cast<float*>(stg + 6 * n);
  a.g = c->slot_grad(gb);
  a.n = n;
  a.n_decay = c->lay[x].n_decay;
  a.sched = c->k2_sched_hyb;
  CKC(c, kern::adamw_split(a, c->hyb_k));
  c->hyb_updates++;
  CKC(c, cudaEventRecord(c->ev_stg_k2[i], c->hyb_k));
  // the pool buffer is free once K2S has read it
  CKC(c, cudaEventRecord(c->ev_grad_free[gb], c->hyb_k));
  const int64_t g1 = ++c->gen;
  c->gradfree_gen[gb] = g1;
  c->gradfree_pub[gb].store(g1);
  release_grad_buffer(c, gb);
  // write-back: hi from the slot, [lo | m | v] from the staging buffer (contiguous in the host block)
  CKC(c, cudaStreamWaitEvent(c->hyb_out, c->ev_stg_k2[i], 0));
  CKC(c, cudaMemcpyAsync(c->h_shadow[x], a.hi, 2 * n, cudaMemcpyDeviceToHost, c->hyb_out));
  CKC(c, cudaMemcpyAsync(c->h_lo[x], stg, 10 * n, cudaMemcpyDeviceToHost, c->hyb_out));
  CKC(c, cudaEventRecord(c->ev_stg_free[i], c->hyb_out));
  // the slot's param half may be refilled (and the next FP of x may run) only after the write-back read it
  CKC(c, cudaEventRecord(c->ev_param_free[s], c->hyb_out));
  CKC(c, cudaEventRecord(c->ev_arrive[x], c->hyb_out));
  const int64_t g2 = ++c->gen;
  c->arrive_gen[x] = g2;
  c->arrive_by_issuer[x] = 0;
  c->arrive_pub[x].store(g2);
  CKC(c, cudaLaunchHostFunc(c->hyb_out, hyb_done_cb, new HybDone{c, x, c->step}));
  c->d2h_bytes += 12 * n;
  c->hyb_d2h += 12 * n;
  c->d2h_copies += 2;
  return SH_OK;
}

// D2H issuer thread: offload pending host-layer gradients, lowest layer first, one per free landing
// buffer; K3 (the layer's sum of squares, needed by sh_step) is enqueued for every pending layer in
// backward order as soon as it is posted, before any wait for a landing buffer.
void d2h_pump(sh_ctx* c) {
  static const bool dbg = getenv("SH_DEBUG_PUMP") != nullptr;
  for (;;) {
    std::vector<sh_ctx::PendD2H*> k3todo;
    {
      std::lock_guard<std::mutex> g(c->dmu);
      for (auto& p : c->pend)
        if (!p.k3_done) k3todo.push_back(&p);  // deque elements do not move on push_back
    }
    if (dbg && !k3todo.empty()) fprintf(stderr, "[pump %.1f] k3 x%zu first L%d\n", now_ms(), k3todo.size(), k3todo[0]->x);
    for (auto* p : k3todo) {
      if (p->k3_on_d2h) {  // on its own stream so the copy engine does not queue behind it
        ProfSet* P = static_cast<ProfSet*>(p->prof);
        CKA(c, cudaStreamWaitEvent(c->k3s, p->ready, 0));
        if (P) CKA(c, cudaEventRecord(P->k30[p->x], c->k3s));
        CKA(c, kern::sumsq(c->slot_grad(p->b), c->lay[p->x].n_pad, c->scratch_d2h, c->partials + p->x, c->k3s));
        if (P) {
          CKA(c, cudaEventRecord(P->k31[p->x], c->k3s));
          P->rec_k3[p->x] = 1;
        }
        CKA(c, cudaEventRecord(c->ev_k3_buf[p->b], c->k3s));
        CKA(c, cudaEventRecord(c->ev_k3_last, c->k3s));
        c->k3_pub.store(p->gen);
      }
      p->k3_done = true;
      c->pend_k3.fetch_add(1);
    }
    if (!k3todo.empty()) notify_state(c);
    {
      std::lock_guard<std::mutex> g(c->dmu);
      if (c->pend.empty()) return;
    }
    // a free landing buffer, or new posts whose K3 must go out first
    if (dbg) fprintf(stderr, "[pump %.1f] wait landing (free %zu)\n", now_ms(), c->land_free.size());
    if (!state_wait(c, [&] { return !c->land_free.empty() || c->pend_posted.load() > c->pend_k3.load(); },
                    "host landing buffer")) {
      std::lock_guard<std::mutex> g(c->dmu);
      for (auto& p : c->pend) c->gradfree_pub[p.b].store(kInf);
      c->pend.clear();
      notify_state(c);
      return;
    }
    int k = -1;
    {
      std::lock_guard<std::mutex> g(c->smu);
      if (c->land_free.empty()) continue;  // woken for K3s
      k = c->land_free.front();
      c->land_free.pop_front();
    }
    sh_ctx::PendD2H p{};
    {
      std::lock_guard<std::mutex> g(c->dmu);
      // lowest layer first among the layers whose gradients are COMPUTED (the driver posts layers well
      // ahead of the GPU: offloading the lowest posted one would park the copy engine behind that
      // layer's backward while earlier gradients wait), else the earliest posted -- except with a shared
      // store, where a slice update needs every rank's offload of the layer: all ranks then keep the
      // backward (POST) order, so the landing buffers every rank holds always wait for the same layers
      auto best = c->pend.end();
      bool best_ready = false;
      for (auto it = c->pend.begin(); it != c->pend.end(); ++it) {
        if (!it->k3_done) continue;
        if (c->shared || c->d2h_fifo) {
          best = it;
          break;
        }
        const bool ready = cudaEventQuery(it->ready) == cudaSuccess;
        if (!ready) cudaGetLastError();
        if (best == c->pend.end()) {
          best = it, best_ready = ready;  // the earliest posted (deque order)
          continue;
        }
        if (ready && (!best_ready || it->step < best->step || (it->step == best->step && it->x < best->x)))
          best = it, best_ready = true;
      }
      if (best == c->pend.end()) {  // only fresh posts: their K3 first
        std::lock_guard<std::mutex> g2(c->smu);
        c->land_free.push_front(k);
        continue;
      }
      p = *best;
      c->pend.erase(best);
    }
    maybe_delay(c->cfg.flags);
    if (dbg) fprintf(stderr, "[pump %.1f] d2h L%d landing %d\n", now_ms(), p.x, k);
    ProfSet* P = static_cast<ProfSet*>(p.prof);
    const int x = p.x;
    c->landing_owner[k] = x;
    c->last_landing[x] = k;
    float* src = c->slot_grad(p.b);
    CKA(c, cudaStreamWaitEvent(c->d2h, p.ready, 0));
    if (P) CKA(c, cudaEventRecord(P->g2c0[x], c->d2h));
    CKA(c, cudaMemcpyAsync(c->landing[k] + p.lo, src + p.lo, 4 * (p.hi - p.lo), cudaMemcpyDeviceToHost, c->d2h));
    if (P) {
      CKA(c, cudaEventRecord(P->g2c1[x], c->d2h));
      P->rec_g2c[x] = 1;
    }
    // the buffer is reusable after the copy and this layer's K3
    if (p.k3_on_d2h) CKA(c, cudaStreamWaitEvent(c->d2h, c->ev_k3_buf[p.b], 0));
    CKA(c, cudaEventRecord(c->ev_grad_free[p.b], c->d2h));
    CKA(c, cudaLaunchHostFunc(c->d2h, landed_cb, new Landed{c, x, p.step, k, p.sc}));
    c->d2h_bytes += 4 * (p.hi - p.lo);
    c->d2h_copies++;
    c->gradfree_pub[p.b].store(p.gen);
    release_grad_buffer(c, p.b);
  }
}

}  // namespace

// =============================================================================== C ABI
extern "C" {

int32_t sh_abi_version(void) { return SH_ABI_VERSION; }
int64_t sh_kernel_launches(void) { return kern::launches(); }
const char* sh_last_error(void) { return sh::last_error_cstr(); }

sh_status sh_nccl_get_unique_id(void* out128) {
  clear_error();
  if (!out128) return SH_ERR_INVALID;
  if (!g_nccl.load()) {
    set_error("libnccl.so.2 not loadable");
    return SH_ERR_UNSUPPORTED;
  }
  ncclUniqueId id;
  if (g_nccl.GetUniqueId(&id) != ncclSuccess) {
    set_error("ncclGetUniqueId failed");
    return SH_ERR_NCCL;
  }
  std::memcpy(out128, &id, sizeof(id));
  return SH_OK;
}

sh_status sh_adam_scalars_for(double lr, double beta1, double beta2, double eps, double weight_decay,
                              int64_t t, sh_adam_scalars* o) {
  if (!o || t < 1) {
    set_error("sh_adam_scalars_for: t must be >= 1");
    return SH_ERR_INVALID;
  }
  const double bc1 = 1.0 - std::pow(beta1, (double)t);
  const double bc2 = 1.0 - std::pow(beta2, (double)t);
  o->beta1 = (float)beta1;
  o->beta2 = (float)beta2;
  o->omb1 = (float)(1.0 - beta1);
  o->omb2 = (float)(1.0 - beta2);
  o->eps = (float)eps;
  o->step_size = (float)(lr / bc1);
  o->sqrt_bc2 = (float)std::sqrt(bc2);
  o->decay = (float)(1.0 - lr * weight_decay);
  return SH_OK;
}

sh_status sh_init(const sh_config* cfg, sh_ctx** out) {
  clear_error();
  if (!cfg || !out) {
    set_error("sh_init: null argument");
    return SH_ERR_INVALID;
  }
  *out = nullptr;
  if (cfg->n_layers < 1 || !cfg->layers) {
    set_error("sh_init: n_layers must be >= 1 with a layers array");
    return SH_ERR_INVALID;
  }
  if (cfg->window < -1 || cfg->window > cfg->n_layers) {
    set_error("sh_init: window %d outside -1..n_layers (%d)", cfg->window, cfg->n_layers);
    return SH_ERR_INVALID;
  }
  if (cfg->precision != SH_FP32 && cfg->precision != SH_BF16_MIXED) {
    set_error("sh_init: unknown precision %d", cfg->precision);
    return SH_ERR_INVALID;
  }
  if (!cfg->compute_stream) {
    set_error("sh_init: compute_stream is required (the caller's cudaStream_t)");
    return SH_ERR_INVALID;
  }
  const int W = cfg->world_size < 1 ? 1 : cfg->world_size;
  const bool dp = W > 1 || (cfg->flags & SH_FLAG_TEST_DP_PATH);
  const bool test_coll = cfg->flags & (SH_FLAG_TEST_NO_COLLECTIVE | SH_FLAG_TEST_HOST_COLLECTIVE);
  if (dp && ((!cfg->nccl_unique_id && !test_coll) || cfg->rank < 0 || cfg->rank >= W)) {
    set_error("sh_init: world_size > 1 needs nccl_unique_id and 0 <= rank < world_size");
    return SH_ERR_INVALID;
  }
  if (cfg->n_executors < 0 || cfg->n_executors > kern::kMaxExecutors) {
    set_error("sh_init: n_executors %d outside 0..%d", cfg->n_executors, kern::kMaxExecutors);
    return SH_ERR_INVALID;
  }
  auto c = std::make_unique<sh_ctx>();
  c->cfg = *cfg;
  c->K = cfg->n_executors > 1 ? cfg->n_executors : 1;
  c->L = cfg->n_layers;
  c->W = W;
  c->rank = cfg->rank;
  c->dp = dp;
  {
    const char* e = getenv("SH_D2H_ORDER");
    c->d2h_fifo = e && strcmp(e, "fifo") == 0;
  }
  c->no_collective = dp && (cfg->flags & SH_FLAG_TEST_NO_COLLECTIVE);
  c->host_coll = dp && !c->no_collective && (cfg->flags & SH_FLAG_TEST_HOST_COLLECTIVE);
  c->use_nccl = dp && !c->no_collective && !c->host_coll;
  c->shared = dp && cfg->shm_name && cfg->shm_name[0];
  c->rs_host = c->shared && (c->use_nccl || c->host_coll);
  if (c->host_coll && (!c->shared || W > kMaxHostCollRanks)) {
    set_error("sh_init: SH_FLAG_TEST_HOST_COLLECTIVE needs shm_name (the shared segment) and world_size <= %d",
              kMaxHostCollRanks);
    return SH_ERR_INVALID;
  }
  if (c->shared) c->shm_name = cfg->shm_name;
  c->bf16 = cfg->precision == SH_BF16_MIXED;
  c->cb = c->bf16 ? 2 : 4;
  c->clip = cfg->max_grad_norm > 0.0f;
  c->warmup = cfg->warmup_steps > 0 ? cfg->warmup_steps : 5;
  c->lr = cfg->lr;
  c->lay.resize(c->L);
  for (int i = 0; i < c->L; ++i) {
    if (!make_layout(cfg->layers[i], &c->lay[i])) return SH_ERR_INVALID;
    c->max_pad = std::max(c->max_pad, c->lay[i].n_pad);
  }
  if (!make_layout(cfg->resident, &c->res)) return SH_ERR_INVALID;
  // data parallel slices: equal length cs = ceil(n_pad / W) rounded to kPad (an in-place
  // all-gather needs equal counts), so slots hold W * cs elements
  c->cs_max = align_up((c->max_pad + W - 1) / W, kPad);
  const int64_t slot_elems = W > 1 ? std::max(c->max_pad, (int64_t)W * c->cs_max) : c->max_pad;
  c->slot_param_bytes = align_up((int64_t)c->cb * slot_elems, 256);
  c->slot_grad_bytes = align_up(4 * slot_elems, 256);
  c->slot_bytes = c->slot_param_bytes + c->slot_grad_bytes;
  const int w0 = cfg->window >= 0 ? cfg->window
                                   : std::min(cfg->warmup_window > 0 ? cfg->warmup_window : 2, c->L);
  c->autotune_pending = cfg->window < 0;
  c->D = cfg->grad_ring_depth > 0 ? cfg->grad_ring_depth : c->L;
  if (c->clip && c->D < c->L) {
    set_error("sh_init: clip mode needs grad_ring_depth 0 (one landing buffer per layer): "
              "every host gradient must be stored until the global norm is known");
    return SH_ERR_INVALID;
  }

  CKC(c.get(), cudaSetDevice(cfg->device));
  c->cs = static_cast<cudaStream_t>(cfg->compute_stream);
  CKC(c.get(), cudaStreamCreateWithFlags(&c->h2d, cudaStreamNonBlocking));
  CKC(c.get(), cudaStreamCreateWithFlags(&c->d2h, cudaStreamNonBlocking));
  {
    // K3 (host layers' Σg², beside the offload) and K1 (restage ahead of a layer's backward) are short
    // HBM-bound launches that run beside the compute stream's GEMMs: at the greatest stream priority
    // their blocks are scheduled as SMs free up instead of queueing behind a GEMM's remaining tiles
    // (SH_SIDE_PRIO=0: default priority, the round-1 behaviour)
    int lo = 0, hi = 0;
    const char* e = getenv("SH_SIDE_PRIO");
    if (!(e && atoi(e) == 0)) CKC(c.get(), cudaDeviceGetStreamPriorityRange(&lo, &hi));
    CKC(c.get(), cudaStreamCreateWithPriority(&c->k3s, cudaStreamNonBlocking, hi));
    CKC(c.get(), cudaStreamCreateWithPriority(&c->stage, cudaStreamNonBlocking, hi));
  }
  CKC(c.get(), cudaEventCreateWithFlags(&c->ev_cs_mark, cudaEventDisableTiming));
  CKC(c.get(), cudaEventCreateWithFlags(&c->ev_comm_done, cudaEventDisableTiming));
  CKC(c.get(), cudaEventCreateWithFlags(&c->ev_k3_last, cudaEventDisableTiming));
  for (int i = 0; i < 2; ++i) {
    CKC(c.get(), cudaEventCreateWithFlags(&c->ev_res_k3[i], cudaEventDisableTiming));
    CKC(c.get(), cudaEventCreateWithFlags(&c->ev_norm[i], cudaEventDisableTiming));
  }
  if (dp) CKC(c.get(), cudaStreamCreateWithFlags(&c->comm, cudaStreamNonBlocking));
  if (c->use_nccl) {
    if (!g_nccl.load()) {
      set_error("sh_init: world_size > 1 but libnccl.so.2 cannot be loaded");
      return SH_ERR_UNSUPPORTED;
    }
    ncclUniqueId id;
    std::memcpy(&id, cfg->nccl_unique_id, sizeof(id));
    sh_status s = nccl_check(c.get(), g_nccl.CommInitRank(&c->nccl, W, id, cfg->rank), "ncclCommInitRank");
    if (s != SH_OK) return s;
  }
  c->slice_fetch = dp && (cfg->flags & SH_FLAG_SLICE_FETCH) && cfg->shm_name && cfg->shm_name[0];
  if (c->slice_fetch && c->use_nccl) {
    if (!g_nccl.AllGather || !g_nccl.CommSplit) {
      set_error("sh_init: SH_FLAG_SLICE_FETCH needs ncclAllGather and ncclCommSplit");
      return SH_ERR_UNSUPPORTED;
    }
    sh_status s = nccl_check(c.get(), g_nccl.CommSplit(c->nccl, 0, cfg->rank, &c->nccl_fetch, nullptr),
                             "ncclCommSplit(fetch)");
    if (s != SH_OK) return s;
  }

  // ---- host store: per layer master | m | v | shadow, plus landing buffers, 2 MiB aligned
  {  // NUMA plan (numa.cpp): topology, the GPU's node, per-layer / landing / slice / worker nodes
    const numa::Topology& topo = numa::topology();
    c->numa_nodes = (int)topo.node_ids.size();
    c->numa_gpu = numa::gpu_node_index(cfg->device);
    if (cfg->numa_policy < SH_NUMA_AUTO || cfg->numa_policy > SH_NUMA_NONE) {
      set_error("sh_init: numa_policy %d is not one of SH_NUMA_*", cfg->numa_policy);
      return SH_ERR_INVALID;
    }
    c->numa_policy = numa::resolve_policy(cfg->numa_policy, c->numa_nodes, dp);
    c->layer_node.assign(c->L, numa::kNone);
    for (int x = 0; x < c->L; ++x) c->layer_node[x] = numa::plan_node(c->numa_policy, x, c->numa_nodes, c->numa_gpu);
    c->land_node = c->numa_policy == SH_NUMA_SPLIT ? numa::plan_node(SH_NUMA_INTERLEAVE, 0, c->numa_nodes, 0)
                                                    : numa::plan_node(c->numa_policy, 0, c->numa_nodes, c->numa_gpu);
    if (c->shared && c->numa_policy != SH_NUMA_NONE) {
      // rank r drives device (device - rank + r): one process per GPU in device order, as launched
      // by torchrun / bench.py.  Under LOCAL slice r lives on its GPU's node; otherwise as planned.
      int n_dev = 0;
      if (cudaGetDeviceCount(&n_dev) != cudaSuccess) cudaGetLastError();
      c->slice_node.assign(c->W, numa::kNone);
      for (int r = 0; r < c->W; ++r) {
        const int dev = cfg->device - cfg->rank + r;
        const int gn = (dev >= 0 && dev < n_dev) ? numa::gpu_node_index(dev) : 0;
        c->slice_node[r] = numa::plan_node(c->numa_policy, r, c->numa_nodes, gn);
      }
    }
    int dflt = (int)std::thread::hardware_concurrency();
    if (c->numa_policy == SH_NUMA_LOCAL && c->numa_nodes > 1 && !topo.cpus[c->numa_gpu].empty())
      dflt = (int)topo.cpus[c->numa_gpu].size();  // LOCAL: the GPU node's cores
    c->n_threads = cfg->cpu_threads > 0 ? cfg->cpu_threads : dflt;
    if (c->n_threads < 1) c->n_threads = 1;
    // off by default: a fixed-window c4max A/B on a slow-D2H box gave +0.6 % with 12 of 16 workers
    // (5.25 / 5.24 vs 5.21 / 5.22 samples/s), inside the autotuned runs' box-to-box noise
    // (profiles/r02_ab_c4max_throttle.txt)
    if (const char* e = getenv("SH_CPU_THROTTLE")) c->cpu_throttle = std::max(0, atoi(e));
    c->worker_node.assign(c->n_threads, numa::kNone);
    for (int t = 0; t < c->n_threads; ++t)
      c->worker_node[t] = numa::worker_node(c->numa_policy, t, c->n_threads, c->numa_gpu);
  }
  c->shadow = c->bf16 && !(cfg->flags & SH_FLAG_FETCH_FP32) && (cfg->flags & SH_FLAG_BF16_SHADOW);
  c->split = c->bf16 && !(cfg->flags & SH_FLAG_FETCH_FP32) && !(cfg->flags & SH_FLAG_BF16_SHADOW);
  c->hblocks.assign(c->L, {});
  c->hshadow.assign(c->L, {});
  c->spilled.assign(c->L, 0);
  if (cfg->spill_dir && cfg->spill_dir[0]) {
    if (c->shared) {
      set_error("sh_init: spill_dir is not supported with a shared (multi-rank) host store");
      return SH_ERR_INVALID;
    }
    struct stat sb;
    if (stat(cfg->spill_dir, &sb) != 0 || !S_ISDIR(sb.st_mode)) {
      set_error("sh_init: spill_dir %s is not a directory", cfg->spill_dir);
      return SH_ERR_INVALID;
    }
    c->spill_dir = cfg->spill_dir;
  }
  c->pin_budget = cfg->host_pin_budget_bytes > 0 ? cfg->host_pin_budget_bytes : 0;
  c->h_master.assign(c->L, nullptr);
  c->h_m.assign(c->L, nullptr);
  c->h_v.assign(c->L, nullptr);
  c->h_shadow.assign(c->L, nullptr);
  c->h_lo.assign(c->L, nullptr);
  {
    const int64_t lb = align_up(4 * c->max_pad, 4096);
    const size_t bytes = align_up((int64_t)c->D * lb + 4096, 1 << 21);
    char* p = nullptr;
    sh_status st = host_block_alloc(bytes, c->n_threads, &p, c->land_node, &c->numa_bound);
    if (st != SH_OK) return st;
    c->hland = {p, bytes};
    c->host_bytes += bytes;
    c->landing.resize(c->D);
    for (int k = 0; k < c->D; ++k) c->landing[k] = reinterpret_cast<float*>(p + (int64_t)k * lb);
    c->h_coef = reinterpret_cast<float*>(p + (int64_t)c->D * lb);
  }
  // rank slices (multiples of kPad so every chunk stays 16-element aligned)
  c->slo.assign(c->L, 0);
  c->shi.assign(c->L, 0);
  for (int x = 0; x < c->L; ++x) {
    const int64_t n = c->lay[x].n_pad;
    if (c->shared) {
      const int64_t cs = align_up((n + c->W - 1) / c->W, kPad);
      c->slo[x] = std::min(n, (int64_t)c->rank * cs);
      c->shi[x] = std::min(n, (int64_t)(c->rank + 1) * cs);
    } else {
      c->slo[x] = 0;
      c->shi[x] = n;
    }
  }
  if (c->host_coll) {  // contribution segment [W][hc_count] + a private result buffer
    c->hc_count = align_up(std::max({(int64_t)W * c->cs_max, c->res.n_pad, 2 * (int64_t)(c->L + 1)}), 1024);
    c->hc_bytes = align_up((int64_t)W * c->hc_count * 4, 1 << 21);
    char* p = nullptr;
    sh_status st = host_block_alloc(c->hc_bytes, c->n_threads, &p);
    if (st != SH_OK) return st;
    c->hc_tmp = reinterpret_cast<float*>(p);
  }
  if (c->shared) {
    // control block: rank 0 creates it, the others wait for it; then every layer segment
    c->ctl_bytes = align_up(sizeof(ShmCtl) + 16 * (int64_t)c->L, 4096);
    char* p = nullptr;
    if (c->rank == 0) {
      sh_status st = shm_map(c.get(), shm_path(c.get(), "ctl"), c->ctl_bytes, true, &p, false);
      if (st != SH_OK) return st;
      std::memset(p, 0, c->ctl_bytes);
      c->ctl = reinterpret_cast<ShmCtl*>(p);
      if (c->host_coll) {
        sh_status st = shm_map(c.get(), shm_path(c.get(), "hc"), c->hc_bytes, true, &p, true);
        if (st != SH_OK) return st;
        c->hc_seg = reinterpret_cast<float*>(p);
      }
      for (int x = 0; x < c->L; ++x) {
        sh_status st2 = ensure_host_layer(c.get(), x);
        if (st2 != SH_OK) return st2;
      }
      c->ctl->magic.store(0x5348u);
      c->ctl->created.store(1);
    } else {
      const double t0 = now_ms();
      for (;;) {  // wait for rank 0's control block and segments
        sh_status st = shm_map(c.get(), shm_path(c.get(), "ctl"), c->ctl_bytes, false, &p, false);
        if (st == SH_OK) {
          c->ctl = reinterpret_cast<ShmCtl*>(p);
          if (c->ctl->created.load() == 1) break;
          munmap(p, c->ctl_bytes);
          c->ctl = nullptr;
        }
        if (now_ms() - t0 > 1e3 * wait_timeout_s()) {
          set_error("shared host store: rank 0 did not create %s", shm_path(c.get(), "ctl").c_str());
          return SH_ERR_STATE;
        }
        usleep(2000);
      }
      if (c->host_coll) {
        sh_status st = shm_map(c.get(), shm_path(c.get(), "hc"), c->hc_bytes, false, &p, true);
        if (st != SH_OK) return st;
        c->hc_seg = reinterpret_cast<float*>(p);
      }
      for (int x = 0; x < c->L; ++x) {
        sh_status st2 = ensure_host_layer(c.get(), x);
        if (st2 != SH_OK) return st2;
      }
    }
    if (!shm_barrier(c.get(), 0, "shared store mapping")) return check_failed(c.get());
    if (c->rank == 0) {  // every rank has it mapped: remove the names (mappings persist)
      shm_unlink(shm_path(c.get(), "ctl").c_str());
      if (c->host_coll) shm_unlink(shm_path(c.get(), "hc").c_str());
      for (int x = 0; x < c->L; ++x) shm_unlink(shm_path(c.get(), "L", x).c_str());
    }
  } else {
    for (int x = w0; x < c->L; ++x) {  // host-optimised layers of the initial window
      sh_status st = ensure_host_layer(c.get(), x);
      if (st != SH_OK) return st;
    }
  }

  // ---- device: resident set, partials, ring, G states
  {
    const int64_t n = c->res.n_pad;
    float* p = nullptr;
    if (cudaMalloc(&p, 16 * n + (int64_t)c->cb * n) != cudaSuccess) {
      cudaGetLastError();
      set_error("sh_init: cudaMalloc of resident set failed");
      return SH_ERR_OOM_DEVICE;
    }
    c->res_master = p;
    c->res_m = p + n;
    c->res_v = p + 2 * n;
    c->res_grad = p + 3 * n;
    c->res_compute = p + 4 * n;
    c->device_bytes += 16 * n + (int64_t)c->cb * n;
    CKC(c.get(), cudaMemset(p, 0, 16 * n + (int64_t)c->cb * n));
    double* d = nullptr;
    const int64_t nd = (c->L + 1) + 3 * (kern::kSumsqMaxBlocks + 1) + 1;
    if (cudaMalloc(&d, nd * 8 + 64) != cudaSuccess) {
      cudaGetLastError();
      set_error("sh_init: cudaMalloc of scratch failed");
      return SH_ERR_OOM_DEVICE;
    }
    CKC(c.get(), cudaMemset(d, 0, nd * 8 + 64));
    c->partials = d;
    if (c->rs_host) {
      if (cudaMalloc(&c->partials_all, 8 * (int64_t)W * (c->L + 1)) != cudaSuccess) {
        cudaGetLastError();
        set_error("sh_init: cudaMalloc of the gathered norm partials failed");
        return SH_ERR_OOM_DEVICE;
      }
      CKC(c.get(), cudaMemset(c->partials_all, 0, 8 * (int64_t)W * (c->L + 1)));
    }
    c->scratch_cs = d + (c->L + 1);
    c->scratch_comm = c->scratch_cs + kern::kSumsqMaxBlocks + 1;
    c->scratch_d2h = c->scratch_comm + kern::kSumsqMaxBlocks + 1;
    c->norm_dev = c->scratch_d2h + kern::kSumsqMaxBlocks + 1;
    c->coef_dev = reinterpret_cast<float*>(c->norm_dev + 1);
    if (kern::k2_dynamic()) {  // in the 64-B slack after coef_dev (zeroed above)
      c->k2_sched_cs = reinterpret_cast<unsigned int*>(c->norm_dev + 2);
      c->k2_sched_comm = c->k2_sched_cs + 2;
    }
    c->k2_sched_hyb = reinterpret_cast<unsigned int*>(c->norm_dev + 2) + 4;  // K2S: always dynamic
    for (int e = 1; e < c->K; ++e) {  // executor gradient buffers (one set: K4 runs in stream order)
      float* xg = nullptr;
      float* xr = nullptr;
      if (cudaMalloc(&xg, 4 * c->max_pad) != cudaSuccess || cudaMalloc(&xr, 4 * n) != cudaSuccess) {
        cudaGetLastError();
        if (xg) cudaFree(xg);
        set_error("sh_init: cudaMalloc of executor %d gradient buffers failed", e);
        return SH_ERR_OOM_DEVICE;
      }
      c->xgrad.push_back(xg);
      c->xres.push_back(xr);
      c->device_bytes += 4 * (c->max_pad + n);
    }
  }
  if (c->bf16 && !c->shadow && !c->split) {  // SH_FLAG_FETCH_FP32: fp32 master staging of the fetches (h2d stream)
    if (cudaMalloc(&c->fp32_stage, c->slot_grad_bytes) != cudaSuccess) {
      cudaGetLastError();
      set_error("sh_init: cudaMalloc of the fp32 fetch staging buffer failed");
      return SH_ERR_OOM_DEVICE;
    }
    c->device_bytes += c->slot_grad_bytes;
  }
  c->g.assign(c->L, GState{});
  c->layer_slot.assign(c->L, -1);
  c->ev_arrive.assign(c->L, nullptr);
  for (auto& e : c->ev_arrive) CKC(c.get(), cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  c->ev_upd.assign(c->L, nullptr);
  for (auto& e : c->ev_upd) {
    CKC(c.get(), cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    CKC(c.get(), cudaEventRecord(e, c->cs));  // completed: nothing to wait for yet
  }
  c->arrive_gen.assign(c->L, 0);
  c->compute_waited.assign(c->L, 0);
  c->arrive_by_issuer.assign(c->L, 0);
  c->arrive_pub = std::make_unique<std::atomic<int64_t>[]>(c->L);
  c->ready = std::make_unique<std::atomic<int64_t>[]>(c->L);
  for (int x = 0; x < c->L; ++x) {
    c->arrive_pub[x].store(0);
    c->ready[x].store(0);
  }
  for (int k = 0; k < c->D; ++k) c->land_free.push_back(k);
  c->landing_owner.assign(c->D, -1);
  c->last_landing.assign(c->L, -1);
  c->layer_gb.assign(c->L, -1);
  c->reg_done.assign(c->L, 0);
  c->coef_of_step.assign(2, 1.0f);
  c->coef_step.assign(2, -1);
  for (auto* v : {&c->p_fp, &c->p_bp, &c->p_c2g, &c->p_g2c, &c->p_stage, &c->p_ogpu, &c->p_ocpu})
    v->assign(c->L, 0.0);
  c->p_slot_i.assign(c->L, c->slot_bytes);
  c->p_gstate_i.resize(c->L);
  for (int x = 0; x < c->L; ++x) c->p_gstate_i[x] = 12 * c->lay[x].n_pad;
  for (auto& P : c->prof) {
    sh_status s = prof_alloc(c.get(), P);
    if (s != SH_OK) return s;
  }
  c->w = w0;
  c->k2_layer = !c->clip;
  c->ring_cap = cfg->ring_slots > 0 ? cfg->ring_slots : 0;
  if (cfg->ring_bytes > 0) {
    // NEXT-4 fixed-byte window ("a fixed-size GPU buffer where the number of DNN layers
    // stored can dynamically change ... for DNN models with a heterogeneous layer structure").
    // Slot 0 can hold the largest layer (progress is guaranteed at every position); slot x >= 1 is
    // sized for layer x, in execution order, while the buffer has room -- a window of consecutive
    // layers therefore fits in the slots of any stretch with the same size mix, and the prefetch
    // stops at the first upcoming layer no evictable slot can hold (pre_common), so the number of
    // layers in the buffer follows their sizes.  G layers 0..w-1 are staged into slots 0..w-1,
    // which fit by construction.
    if (c->clip || c->dp || c->autotune_pending || cfg->ring_slots > 0) {
      set_error("sh_init: ring_bytes needs no clipping, a single rank, a fixed window and ring_slots 0");
      return SH_ERR_INVALID;
    }
    auto slot_sz = [&](int64_t cap, int64_t* pb) {
      *pb = align_up((int64_t)c->cb * cap, 256);
      return *pb + align_up(4 * cap, 256);
    };
    int64_t pb = 0, total = slot_sz(c->max_pad, &pb);
    if (total > cfg->ring_bytes) {
      set_error("sh_init: ring_bytes %lld cannot hold the largest layer (%lld B)", (long long)cfg->ring_bytes,
                (long long)total);
      return SH_ERR_INVALID;
    }
    c->slot_off.push_back(0);
    c->slot_cap.push_back(c->max_pad);
    c->slot_pb.push_back(pb);
    for (int x = 1; x < c->L; ++x) {
      const int64_t b = slot_sz(c->lay[x].n_pad, &pb);
      if (total + b > cfg->ring_bytes) break;
      c->slot_off.push_back(total);
      c->slot_cap.push_back(c->lay[x].n_pad);
      c->slot_pb.push_back(pb);
      total += b;
    }
    c->byte_ring_total = total;
  }
  if (cfg->hybrid_layers < 0) {
    set_error("sh_init: hybrid_layers must be >= 0");
    return SH_ERR_INVALID;
  }
  if (cfg->hybrid_layers > 0) {
    // R28 hybrid update (include/sh.h sh_config.hybrid_layers)
    if (!c->split || c->clip || c->dp || c->byte_ring() || (cfg->spill_dir && cfg->spill_dir[0])) {
      set_error("sh_init: hybrid_layers needs the split host master (bf16), no clipping, world_size 1, "
                "no fixed-byte ring and no spill tier");
      return SH_ERR_INVALID;
    }
    c->n_hyb = cfg->hybrid_layers;
    const char* e = getenv("SH_HYB_STAGING");
    const int S = std::max(2, e ? atoi(e) : 3);
    int lo = 0, hi = 0;
    CKC(c.get(), cudaDeviceGetStreamPriorityRange(&lo, &hi));
    CKC(c.get(), cudaStreamCreateWithFlags(&c->hyb_in, cudaStreamNonBlocking));
    CKC(c.get(), cudaStreamCreateWithPriority(&c->hyb_k, cudaStreamNonBlocking, hi));
    CKC(c.get(), cudaStreamCreateWithFlags(&c->hyb_out, cudaStreamNonBlocking));
    for (int i = 0; i < S; ++i) {
      char* p = nullptr;
      if (cudaMalloc(&p, 10 * c->max_pad) != cudaSuccess) {
        cudaGetLastError();
        set_error("sh_init: cudaMalloc of a hybrid-update staging buffer (%lld B) failed", (long long)(10 * c->max_pad));
        return SH_ERR_OOM_DEVICE;
      }
      c->hyb_stg.push_back(p);
      c->device_bytes += 10 * c->max_pad;
      for (auto* v : {&c->ev_stg_in, &c->ev_stg_k2, &c->ev_stg_free}) {
        cudaEvent_t ev = nullptr;
        CKC(c.get(), cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        v->push_back(ev);
      }
      CKC(c.get(), cudaEventRecord(c->ev_stg_free[i], c->hyb_out));  // free: every wait has a completed event
    }
    c->hyb_stg_of.assign(c->L, -1);
    c->hyb_issued.assign(c->L, -1);
  }
  c->n_active = c->ring_for(w0);
  c->d = c->n_active - 1;
  c->layer_gbuf.assign(c->L, -1);
  {
    sh_status s = ensure_gbufs(c.get(), w0);
    if (s != SH_OK) return s;
  }
  {
    sh_status s = alloc_ring(c.get(), c->n_active);
    if (s != SH_OK) return s;
    for (int x = 0; x < w0; ++x) {
      s = alloc_g(c.get(), x);
      if (s != SH_OK) return s;
    }
  }
  CKC(c.get(), cudaDeviceSynchronize());

  c->ih2d.start();
  c->id2h.start();
  for (int t = 0; t < c->n_threads; ++t) {
    sh_ctx* cp = c.get();
    c->workers.emplace_back([cp, t] { worker_loop(cp, t); });
  }
  *out = c.release();
  return SH_OK;
}

sh_status sh_register_host_store(sh_ctx* c, int32_t layer, const float* params, const float* m,
                                 const float* v, int64_t step) {
  clear_error();
  if (!c || !params) {
    set_error("sh_register_host_store: null argument");
    return SH_ERR_INVALID;
  }
  if (c->phase != sh_ctx::IDLE || (c->step > 0 && step != c->step)) {
    set_error("sh_register_host_store: only before the first step (or between steps with step == current)");
    return SH_ERR_STATE;
  }
  if (layer < -1 || layer >= c->L) {
    set_error("sh_register_host_store: layer %d out of range", layer);
    return SH_ERR_INVALID;
  }
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  if (step < 0) step = 0;
  // re-registration after the store is live (resume / state reload between steps): the previous
  // step's CPU updates, prefetches and per-layer K2s may still read or write this layer's state --
  // drain them first; the ring's compute copies are re-staged below
  const bool live = c->registered_all;
  if (live) {
    st = sync_all(c);
    if (st != SH_OK) return st;
  }
  if (layer == -1) {
    const int64_t n = c->res.n_pad;
    std::vector<float> tmp(n);
    pack_layer(c->res, params, tmp.data());
    CKC(c, cudaMemcpy(c->res_master, tmp.data(), 4 * n, cudaMemcpyHostToDevice));
    pack_layer(c->res, m, tmp.data());
    CKC(c, cudaMemcpy(c->res_m, tmp.data(), 4 * n, cudaMemcpyHostToDevice));
    pack_layer(c->res, v, tmp.data());
    CKC(c, cudaMemcpy(c->res_v, tmp.data(), 4 * n, cudaMemcpyHostToDevice));
    if (c->bf16)
      CKC(c, kern::cast_bf16(c->res_master, static_cast<uint16_t*>(c->res_compute), n, c->cs));
    else
      CKC(c, cudaMemcpyAsync(c->res_compute, c->res_master, 4 * n, cudaMemcpyDeviceToDevice, c->cs));
    CKC(c, cudaStreamSynchronize(c->cs));
    c->res_reg = true;
  } else {
    const int x = layer;
    const int64_t n = c->lay[x].n_pad;
    std::vector<float> tmp, mst;
    float *hp = c->h_master[x], *hm = c->h_m[x], *hv = c->h_v[x];
    const bool own = c->hblocks[x].p && !(c->shared && c->rank != 0);  // this rank writes the host copy
    AlignedBuf sbuf(c->spilled[x] ? sp_file_bytes(c, x) : 0);
    if (c->spilled[x]) {  // NEXT-2: staged in the file's layout, written with one O_DIRECT request
      if (!sbuf.p) {
        set_error("sh_register_host_store: no memory for a spill staging copy");
        return SH_ERR_OOM_HOST;
      }
      std::memset(sbuf.p, 0, sp_file_bytes(c, x));
      hp = sbuf.f();
      hm = reinterpret_cast<float*>(sbuf.b() + sp_rb(c, x));
      hv = reinterpret_cast<float*>(sbuf.b() + 2 * sp_rb(c, x));
      if (c->split) {  // region 0 holds [hi | lo]: the fp32 master goes through a temporary
        mst.resize(n);
        hp = mst.data();
      }
    } else if (!own) {  // no (own) host copy to write: stage through a temporary
      tmp.resize(3 * n);
      hp = tmp.data();
      hm = hp + n;
      hv = hp + 2 * n;
    } else if (c->split) {  // split master: the fp32 master through a temporary, m / v in place
      mst.resize(n);
      hp = mst.data();
    }
    pack_layer(c->lay[x], params, hp);
    pack_layer(c->lay[x], m, hm);
    pack_layer(c->lay[x], v, hv);
    if (c->shadow && c->h_shadow[x] && hp == c->h_master[x]) cpu::cast_bf16_range(hp, c->h_shadow[x], 0, n);
    if (c->split && own) split_par(c, hp, c->h_shadow[x], c->h_lo[x], 0, n);
    if (c->spilled[x]) {
      if (c->shadow) cpu::cast_bf16_range(hp, reinterpret_cast<uint16_t*>(sbuf.b() + 3 * sp_rb(c, x)), 0, n);
      if (c->split) {
        uint16_t* h16 = reinterpret_cast<uint16_t*>(sbuf.b());
        split_par(c, hp, h16, h16 + n, 0, n);
      }
      st = spill_file_io(c, true, x, sbuf.p, sp_file_bytes(c, x));
      if (st != SH_OK) return st;
    }
    c->ready[x].store(step);
    if (c->shared && c->rank == 0) {
      c->ctl->cnt[x].store((int64_t)c->W * step);
      c->ctl->cnt[c->L + x].store((int64_t)c->W * step);
    }
    if (c->is_g(x)) {
      CKC(c, cudaMemcpy(c->g[x].master, hp, 4 * n, cudaMemcpyHostToDevice));
      CKC(c, cudaMemcpy(c->g[x].m, hm, 4 * n, cudaMemcpyHostToDevice));
      CKC(c, cudaMemcpy(c->g[x].v, hv, 4 * n, cudaMemcpyHostToDevice));
    }
    c->reg_done[x] = 1;
  }
  c->step = step;
  bool all = c->res_reg;
  for (int x = 0; x < c->L; ++x) all = all && c->reg_done[x];
  if (all && !c->registered_all) {
    if (!shm_barrier(c, 1, "registration of the shared host store")) return check_failed(c);
    c->registered_all = true;
    st = stage_g_layers(c);
    if (st != SH_OK) return st;
    CKC(c, cudaStreamSynchronize(c->cs));
  } else if (live && layer >= 0) {
    // every ring copy of the layer is stale: drop the host-layer mapping (the next use fetches
    // the new state) and re-stage the GPU-optimised layers from their (new) HBM masters
    st = stage_g_layers(c);
    if (st != SH_OK) return st;
    CKC(c, cudaStreamSynchronize(c->cs));
  }
  return SH_OK;
}

sh_status sh_set_lr(sh_ctx* c, double lr) {
  if (!c) return SH_ERR_INVALID;
  c->lr = lr;
  return SH_OK;
}

sh_status sh_forward_layer(sh_ctx* c, int32_t x, int32_t phase, void** dev_params) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  const double t0 = now_ms();
  if (phase == SH_PRE) {
    const bool start = c->phase == sh_ctx::IDLE && x == 0;
    const bool cont = c->phase == sh_ctx::FP && c->last_hook == SH_POST && x == c->last_layer + 1;
    if (!(start || cont) || !dev_params) {
      set_error("sh_forward_layer(%d, PRE) out of order (phase %d, last layer %d)", x, (int)c->phase, c->last_layer);
      return SH_ERR_STATE;
    }
    if (start) {
      if (!c->registered_all) {
        set_error("sh_forward_layer: register every layer and the resident set first");
        return SH_ERR_STATE;
      }
      // harvest the profile of step-2 (its issuer work is complete by the ready chain)
      prof_harvest(c, c->prof[c->step & 1]);
      if (step_profiled(c, c->step)) {
        ProfSet& P = c->prof[c->step & 1];
        prof_reset(c, P, c->step);
        CKC(c, cudaEventRecord(P.t0, c->cs));
        CKC(c, cudaLaunchHostFunc(c->cs, t0_cb, &P));
        P.rec_t0 = true;
      }
      CKC(c, cudaMemsetAsync(c->res_grad, 0, 4 * c->res.n_pad, c->cs));
      for (float* xr : c->xres) CKC(c, cudaMemsetAsync(xr, 0, 4 * c->res.n_pad, c->cs));
      c->phase = sh_ctx::FP;
    }
    st = pre_common(c, x, x);
    if (st != SH_OK) return st;
    if (ProfSet* P = cur_prof(c)) {
      CKC(c, cudaEventRecord(P->fp0[x], c->cs));
    }
    fill_param_ptrs(c, x, dev_params);
    c->last_layer = x;
    c->last_hook = SH_PRE;
  } else if (phase == SH_POST) {
    if (!(c->phase == sh_ctx::FP && c->last_hook == SH_PRE && x == c->last_layer)) {
      set_error("sh_forward_layer(%d, POST) out of order", x);
      return SH_ERR_STATE;
    }
    if (ProfSet* P = cur_prof(c)) {
      CKC(c, cudaEventRecord(P->fp1[x], c->cs));
      P->rec_fp[x] = 1;
    }
    CKC(c, cudaEventRecord(c->ev_param_free[c->layer_slot[x]], c->cs));
    c->last_hook = SH_POST;
  } else {
    set_error("sh_forward_layer: bad phase %d", phase);
    return SH_ERR_INVALID;
  }
  c->t_async_ms += now_ms() - t0;
  c->n_async++;
  return SH_OK;
}

sh_status sh_backward_layer(sh_ctx* c, int32_t x, int32_t phase, void** dev_params, float** dev_grads) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  const double t0 = now_ms();
  const int L = c->L;
  if (phase == SH_PRE) {
    const bool start = c->phase == sh_ctx::FP && c->last_hook == SH_POST && c->last_layer == L - 1 && x == L - 1;
    const bool cont = c->phase == sh_ctx::BP && c->last_hook == SH_POST && x == c->last_layer - 1;
    if (!(start || cont) || !dev_params || !dev_grads) {
      set_error("sh_backward_layer(%d, PRE) out of order (phase %d, last layer %d)", x, (int)c->phase, c->last_layer);
      return SH_ERR_STATE;
    }
    if (start) {
      c->phase = sh_ctx::BP;
      // per-step Adam scalars: fixed once BP starts (the CPU updates begin during BP)
      st = sh_adam_scalars_for(c->lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, c->cfg.weight_decay,
                               c->step + 1, &c->sc);
      if (st != SH_OK) return st;
    }
    const int pos = 2 * L - 1 - x;
    st = pre_common(c, x, pos);
    if (st != SH_OK) return st;
    if (c->n_hyb > 0) {
      st = hyb_issue(c, x);
      if (st != SH_OK) return st;
    }
    float* gdst = nullptr;
    if (c->is_g(x) && c->k2_layer) {
      // dedicated grad buffer: no wait on this slot's pending offload
      const int b = (int)(c->gbuf_rr++ % (int64_t)c->gbuf.size());
      c->layer_gbuf[x] = b;
      c->gbuf_owner[b] = x;
      CKC(c, cudaStreamWaitEvent(c->cs, c->ev_gbuf_free[b], 0));  // its previous K2 consumed it
      gdst = c->gbuf[b];
    } else {
      // any free buffer of the gradient pool (its previous offload issued; the GPU waits for it)
      const int64_t need_n = c->rs_host && !c->is_g(x)
                                 ? (int64_t)c->W * align_up((c->lay[x].n_pad + c->W - 1) / c->W, kPad)
                                 : c->lay[x].n_pad;
      const int b = take_grad_buffer(c, x, need_n);
      if (b < 0) return check_failed(c);
      c->layer_gb[x] = b;
      if (c->gradfree_gen[b] > c->gradfree_waited[b]) {
        CKC(c, cudaStreamWaitEvent(c->cs, c->ev_grad_free[b], 0));
        c->gradfree_waited[b] = c->gradfree_gen[b];
      }
      gdst = c->slot_grad(b);
    }
    // (a reduce-scattered host layer spans W equal slices: zero the padding past n_pad too)
    const int64_t zn = c->rs_host && !c->is_g(x)
                           ? std::max(c->lay[x].n_pad, (int64_t)c->W * align_up((c->lay[x].n_pad + c->W - 1) / c->W, kPad))
                           : c->lay[x].n_pad;
    CKC(c, cudaMemsetAsync(gdst, 0, 4 * zn, c->cs));
    for (float* xg : c->xgrad) CKC(c, cudaMemsetAsync(xg, 0, 4 * c->lay[x].n_pad, c->cs));
    c->cur_gdst = gdst;
    if (ProfSet* P = cur_prof(c)) CKC(c, cudaEventRecord(P->bp0[x], c->cs));
    fill_param_ptrs(c, x, dev_params);
    const LayerLayout& Lx = c->lay[x];
    for (int k = 0; k < Lx.n_tensors; ++k) dev_grads[k] = gdst + Lx.offset[k];
    c->last_layer = x;
    c->last_hook = SH_PRE;
  } else if (phase == SH_POST) {
    if (!(c->phase == sh_ctx::BP && c->last_hook == SH_PRE && x == c->last_layer)) {
      set_error("sh_backward_layer(%d, POST) out of order", x);
      return SH_ERR_STATE;
    }
    const int s = c->layer_slot[x];
    const int gb = c->is_g(x) && c->k2_layer ? -1 : c->layer_gb[x];  // gradient-pool buffer
    const int64_t n = c->lay[x].n_pad;
    if (c->K > 1) {  // K4: fold the executors' micro-batch gradients (counted as BP compute)
      st = exec_fold(c, c->cur_gdst, c->xgrad, n);
      if (st != SH_OK) return st;
    }
    ProfSet* P = cur_prof(c);
    if (P) {
      CKC(c, cudaEventRecord(P->bp1[x], c->cs));
      P->rec_bp[x] = 1;
    }
    CKC(c, cudaEventRecord(c->ev_param_free[s], c->cs));
    cudaEvent_t grads_ready = gb >= 0 ? c->ev_grad_done[gb] : nullptr;
    if (c->is_g(x) && c->k2_layer) {
      // GPU-optimised layer, no clipping: grads in its dedicated buffer b; [W>1: all-reduce];
      // K3; per-layer K2 (bitwise the same as a step-end update) on a side stream -- the stage
      // stream (single GPU) or the comm stream (data parallel, in order after the collective) --
      // so the compute stream goes straight on to the next layer.  The next uses of the slot (a
      // fetch into it, the next FP of the layer) and of the buffer wait on events recorded after K2.
      const int b = c->layer_gbuf[x];
      float* gb = c->gbuf[b];
      // (single GPU: on the compute stream -- measured on C4, K2 running beside the next layer's
      // GEMMs slows them by about as much as it saves, and in order its roofline stays clean)
      cudaStream_t ks = c->dp ? c->comm : c->cs;
      if (c->dp) {
        CKC(c, cudaEventRecord(c->ev_gbuf_ready[b], c->cs));
        CKC(c, cudaStreamWaitEvent(c->comm, c->ev_gbuf_ready[b], 0));
        st = coll_allreduce_avg(c, gb, n, c->comm, "ncclAllReduce(layer grads)");
        if (st != SH_OK) return st;
        CKC(c, kern::sumsq(gb, n, c->scratch_comm, c->partials + x, c->comm));
      } else {
        if (P) CKC(c, cudaEventRecord(P->k30[x], c->cs));
        CKC(c, kern::sumsq(gb, n, c->scratch_cs, c->partials + x, c->cs));
        if (P) {
          CKC(c, cudaEventRecord(P->k31[x], c->cs));
          P->rec_k3[x] = 1;
        }
        if (ks != c->cs) {
          CKC(c, cudaEventRecord(c->ev_gbuf_ready[b], c->cs));
          CKC(c, cudaStreamWaitEvent(ks, c->ev_gbuf_ready[b], 0));
        }
      }
      if (P) CKC(c, cudaEventRecord(P->k2l0[x], ks));
      kern::K2Args a{};
      a.sc = c->sc;
      a.coef = nullptr;
      a.out_bf16 = c->bf16;
      a.n_entries = 1;
      a.e[0] = kern::K2Entry{c->g[x].master, c->g[x].m, c->g[x].v, gb, c->slot_param(s), n, c->lay[x].n_decay};
      a.sched = ks == c->cs ? c->k2_sched_cs : c->k2_sched_comm;
      CKC(c, kern::adamw_multi(a, ks));
      if (P) {
        CKC(c, cudaEventRecord(P->k2l1[x], ks));
        P->rec_k2l[x] = 1;
      }
      CKC(c, cudaEventRecord(c->ev_param_free[s], ks));  // param half rewritten by K2
      CKC(c, cudaEventRecord(c->ev_upd[x], ks));
      CKC(c, cudaEventRecord(c->ev_gbuf_free[b], ks));
      CKC(c, cudaEventRecord(c->ev_arrive[x], ks));     // the next FP of x waits for its update
      const int64_t g2 = ++c->gen;
      c->arrive_gen[x] = g2;
      c->arrive_by_issuer[x] = 0;
      c->arrive_pub[x].store(g2);
    } else if (c->dp) {
      // data parallel: average this layer's grads across ranks before the offload (K-e)
      float* g = c->slot_grad(gb);
      CKC(c, cudaEventRecord(c->ev_grad_done[gb], c->cs));
      CKC(c, cudaStreamWaitEvent(c->comm, c->ev_grad_done[gb], 0));
      if (c->rs_host && !c->is_g(x)) {
        // host layer, shared store: this rank offloads only its slice -> reduce-scatter, and the
        // K3 covers the slice (the per-rank partials are folded at sh_step)
        st = coll_reduce_scatter_avg(c, g, x, c->comm);
        if (st != SH_OK) return st;
        CKC(c, kern::sumsq(g + c->slo[x], c->shi[x] - c->slo[x], c->scratch_comm, c->partials + x, c->comm));
      } else {
        st = coll_allreduce_avg(c, g, n, c->comm, "ncclAllReduce(layer grads)");
        if (st != SH_OK) return st;
        CKC(c, kern::sumsq(g, n, c->scratch_comm, c->partials + x, c->comm));
      }
      CKC(c, cudaEventRecord(c->ev_reduced[gb], c->comm));
      grads_ready = c->ev_reduced[gb];
    } else if (c->is_g(x)) {  // clip mode: grads stay in their pool buffer until sh_step's K2
      if (P) CKC(c, cudaEventRecord(P->k30[x], c->cs));
      CKC(c, kern::sumsq(c->slot_grad(gb), n, c->scratch_cs, c->partials + x, c->cs));
      if (P) {
        CKC(c, cudaEventRecord(P->k31[x], c->cs));
        P->rec_k3[x] = 1;
      }
      CKC(c, cudaEventRecord(c->ev_grad_done[gb], c->cs));
    } else if (c->is_hyb(x)) {  // R28: K3 on the compute stream (as for a G layer), then the GPU update
      if (P) CKC(c, cudaEventRecord(P->k30[x], c->cs));
      CKC(c, kern::sumsq(c->slot_grad(gb), n, c->scratch_cs, c->partials + x, c->cs));
      if (P) {
        CKC(c, cudaEventRecord(P->k31[x], c->cs));
        P->rec_k3[x] = 1;
      }
      st = hyb_update(c, x, s, gb);
      if (st != SH_OK) return st;
    } else {
      // host layer: K3 runs on its own stream beside the offload (off the compute stream)
      CKC(c, cudaEventRecord(c->ev_grad_done[gb], c->cs));
    }
    const bool k3_on_d2h = !c->dp && !c->is_g(x);
    if (!c->is_g(x) && !c->is_hyb(x)) {  // post the offload: the D2H scheduler issues it lowest layer first (d2h_pump)
      const int64_t gen = ++c->gen;
      c->gradfree_gen[gb] = gen;
      if (k3_on_d2h) c->k3_last_gen = gen;
      {
        std::lock_guard<std::mutex> g(c->dmu);
        c->pend.push_back(sh_ctx::PendD2H{x, gb, c->step, gen, c->slo[x], c->shi[x], c->sc, P, grads_ready,
                                          k3_on_d2h, false});
      }
      c->pend_posted.fetch_add(1);
      notify_state(c);
      c->id2h.push([c] { d2h_pump(c); });
    }
    c->last_hook = SH_POST;
  } else {
    set_error("sh_backward_layer: bad phase %d", phase);
    return SH_ERR_INVALID;
  }
  c->t_async_ms += now_ms() - t0;
  c->n_async++;
  return SH_OK;
}

sh_status sh_resident(sh_ctx* c, void** dev_params, float** dev_grads) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  for (int k = 0; k < c->res.n_tensors; ++k) {
    if (dev_params) dev_params[k] = static_cast<char*>(c->res_compute) + (int64_t)c->cb * c->res.offset[k];
    if (dev_grads) dev_grads[k] = c->res_grad + c->res.offset[k];
  }
  return SH_OK;
}

sh_status sh_executor_grads(sh_ctx* c, int32_t layer, int32_t executor, float** dev_grads) {
  clear_error();
  if (!c || !dev_grads) return SH_ERR_INVALID;
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  if (executor < 0 || executor >= c->K) {
    set_error("sh_executor_grads: executor %d outside 0..%d", executor, c->K - 1);
    return SH_ERR_INVALID;
  }
  if (layer < 0) {
    float* base = executor == 0 ? c->res_grad : c->xres[executor - 1];
    for (int k = 0; k < c->res.n_tensors; ++k) dev_grads[k] = base + c->res.offset[k];
    return SH_OK;
  }
  if (!(c->phase == sh_ctx::BP && c->last_hook == SH_PRE && layer == c->last_layer)) {
    set_error("sh_executor_grads(%d): layer must be between its backward PRE and POST", layer);
    return SH_ERR_STATE;
  }
  float* base = executor == 0 ? c->cur_gdst : c->xgrad[executor - 1];
  const LayerLayout& Lx = c->lay[layer];
  for (int k = 0; k < Lx.n_tensors; ++k) dev_grads[k] = base + Lx.offset[k];
  return SH_OK;
}

sh_status sh_forward_only_end(sh_ctx* c) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  if (!(c->phase == sh_ctx::FP && c->last_layer == c->L - 1 && c->last_hook == SH_POST)) {
    set_error("sh_forward_only_end: the forward of layer L-1 must be the last hook");
    return SH_ERR_STATE;
  }
  // nothing was updated: every copy in the ring stays valid for the next pass; the step counter
  // (Adam's t) does not advance.  Pending profiling of this pass is dropped.
  ProfSet& P = c->prof[c->step & 1];
  if (P.active && P.step == c->step) P.active = false;
  c->phase = sh_ctx::IDLE;
  c->last_layer = -1;
  c->last_hook = SH_POST;
  c->fwd_passes++;
  return SH_OK;
}

sh_status sh_step(sh_ctx* c, double* grad_norm_out) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  if (!(c->phase == sh_ctx::BP && c->last_layer == 0 && c->last_hook == SH_POST)) {
    set_error("sh_step: the backward of layer 0 must be the last hook before sh_step");
    return SH_ERR_STATE;
  }
  const int L = c->L;
  if (c->K > 1) {
    st = exec_fold(c, c->res_grad, c->xres, c->res.n_pad);
    if (st != SH_OK) return st;
  }
  if (c->dp) {
    // resident grads: average too, on the comm stream after the caller's embedding backward
    CKC(c, cudaEventRecord(c->ev_cs_mark, c->cs));
    CKC(c, cudaStreamWaitEvent(c->comm, c->ev_cs_mark, 0));
    st = coll_allreduce_avg(c, c->res_grad, c->res.n_pad, c->comm, "ncclAllReduce(resident grads)");
    if (st != SH_OK) return st;
    CKC(c, kern::sumsq(c->res_grad, c->res.n_pad, c->scratch_comm, c->partials + L, c->comm));
    st = coll_fold_partials(c, c->comm);
    if (st != SH_OK) return st;
    CKC(c, cudaEventRecord(c->ev_comm_done, c->comm));
    CKC(c, cudaStreamWaitEvent(c->cs, c->ev_comm_done, 0));
  } else {
    CKC(c, kern::sumsq(c->res_grad, c->res.n_pad, c->scratch_cs, c->partials + L, c->cs));
  }
  bool norm_on_d2h = false;
  if (!c->dp && c->w < L && !c->clip) {
    // no clipping: nothing on the compute stream needs the norm.  Finalize it on the D2H stream
    // behind the host layers' K3s, queued on the D2H issuer, so the driver never waits for the
    // issuer (which may be held back by landing-buffer waits) at the step boundary.
    const int par = (int)(c->step & 1);
    CKC(c, cudaEventRecord(c->ev_res_k3[par], c->cs));
    cudaEvent_t rk = c->ev_res_k3[par], nd = c->ev_norm[par];
    const double mx = c->cfg.max_grad_norm;
    c->id2h.push([c, rk, nd, L, mx] {
      CKA(c, cudaStreamWaitEvent(c->d2h, rk, 0));
      CKA(c, cudaStreamWaitEvent(c->d2h, c->ev_k3_last, 0));  // every host layer's K3 (k3 stream)
      CKA(c, kern::norm_finalize(c->partials, L + 1, mx, c->norm_dev, c->coef_dev, c->d2h));
      CKA(c, cudaEventRecord(nd, c->d2h));
    });
    norm_on_d2h = true;
  } else {
    if (!c->dp && c->w < L) {  // clip mode: K2 needs the coefficient -- wait for the last K3
      const int64_t gen = c->k3_last_gen;
      if (!state_wait(c, [&] { return c->k3_pub.load() >= gen; }, "last K3 issue")) return check_failed(c);
      CKC(c, cudaStreamWaitEvent(c->cs, c->ev_k3_last, 0));
    }
    CKC(c, kern::norm_finalize(c->partials, L + 1, c->cfg.max_grad_norm, c->norm_dev, c->coef_dev, c->cs));
  }
  ProfSet* P = cur_prof(c);
  if (P) CKC(c, cudaEventRecord(P->k2a, c->cs));
  kern::K2Args a{};
  a.sc = c->sc;
  a.coef = c->clip ? c->coef_dev : nullptr;
  a.out_bf16 = c->bf16;
  int64_t bytes = 0;
  int launches = 0;
  // clip mode: the GPU-optimised layers (pinned in the ring) are updated here with the clip
  // coefficient, layer 0 first (the next FP starts with it); otherwise they were updated per layer
  for (int x = 0; x < (c->k2_layer ? 0 : c->w); ++x) {
    const int s = c->layer_slot[x];
    if (s < 0) {
      set_error("internal: GPU-optimised layer %d not in the ring at sh_step", x);
      return SH_ERR_STATE;
    }
    a.e[a.n_entries++] = kern::K2Entry{c->g[x].master, c->g[x].m, c->g[x].v, c->slot_grad(c->layer_gb[x]),
                                       c->slot_param(s), c->lay[x].n_pad, c->lay[x].n_decay};
    if (a.n_entries == kern::kK2MaxEntries) {
      st = push_k2(c, a, &bytes, &launches);
      if (st != SH_OK) return st;
    }
  }
  a.e[a.n_entries++] = kern::K2Entry{c->res_master, c->res_m, c->res_v, c->res_grad, c->res_compute,
                                     c->res.n_pad, c->res.n_decay};
  st = push_k2(c, a, &bytes, &launches);
  if (st != SH_OK) return st;
  if (!c->k2_layer)
    for (int x = 0; x < c->w; ++x) {
      CKC(c, cudaEventRecord(c->ev_upd[x], c->cs));
      // clip mode: the layer's pool buffer is free again once this K2 has read it
      const int b = c->layer_gb[x];
      CKC(c, cudaEventRecord(c->ev_grad_free[b], c->cs));
      const int64_t g2 = ++c->gen;
      c->gradfree_gen[b] = g2;
      c->gradfree_pub[b].store(g2);
      release_grad_buffer(c, b);
    }
  if (P) {
    CKC(c, cudaEventRecord(P->k2b, c->cs));
    P->rec_k2 = true;
    P->k2_bytes = bytes;
    P->k2_launches = launches;
  }
  if (c->clip) {
    const int64_t t = c->step;
    CKC(c, cudaMemcpyAsync(c->h_coef + (t & 1), c->coef_dev, 4, cudaMemcpyDeviceToHost, c->cs));
    CKC(c, cudaLaunchHostFunc(c->cs, coef_cb, new CoefMsg{c, t}));
  }
  // host-optimised copies in the ring are stale after this step's CPU update
  for (int s = 0; s < c->n_active; ++s) {
    const int o = c->slot_layer[s];
    if (o >= 0 && !c->is_g(o) && !c->is_hyb(o)) {  // (a hybrid layer's copy is the updated one)
      c->layer_slot[o] = -1;
      c->slot_layer[s] = -1;
    }
  }
  c->step++;
  c->phase = sh_ctx::IDLE;
  c->last_layer = -1;
  c->last_hook = SH_POST;
  if (c->autotune_pending && c->step >= c->warmup) {
    int32_t wout = 0;
    st = sh_autotune_window(c, nullptr, &wout);
    if (st != SH_OK) return st;
  }
  if (grad_norm_out) {
    CKC(c, cudaStreamSynchronize(c->cs));
    if (norm_on_d2h) {
      c->id2h.drain();
      CKC(c, cudaEventSynchronize(c->ev_norm[(c->step - 1) & 1]));
    }
    CKC(c, cudaMemcpy(grad_norm_out, c->norm_dev, 8, cudaMemcpyDeviceToHost));
  }
  return check_failed(c);
}

sh_status sh_synchronize(sh_ctx* c) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  return sync_all(c);
}

sh_status sh_get_profile(sh_ctx* c, sh_profile* o) {
  clear_error();
  if (!c || !o) return SH_ERR_INVALID;
  if (c->phase != sh_ctx::IDLE) {
    set_error("sh_get_profile: only between steps");
    return SH_ERR_STATE;
  }
  sh_status st = sync_all(c);
  if (st != SH_OK) return st;
  // t_c2g of GPU-optimised layers is not observed (they are never fetched): use the bytes
  // rate of the measured host layers (same link, same size class)
  // fetched bytes per element (per layer: fp32 master + K1 cast without a shadow); with
  // SH_FLAG_LATE_SHADOW the host layers will fetch a bf16 shadow after the autotune: solve for that
  const bool late = c->bf16 && (c->cfg.flags & SH_FLAG_LATE_SHADOW) && !c->shared;
  auto fbx = [&](int x) { return (c->bf16 && !has_shadow(c, x)) ? 4.0 : (double)c->cb; };
  double rate = 0;  // ms per byte: mean of the measured fetches
  double rate_min = 0;  // the fastest one: the warm-up runs with most layers on the host, so its
                        // fetches compete with the heaviest CPU-Adam traffic; the tuned run's don't
  int nr = 0;
  for (int x = 0; x < c->L; ++x)
    if (c->p_c2g[x] > 0) {
      const double r = c->p_c2g[x] / (fbx(x) * c->lay[x].n_pad);
      rate += r;
      rate_min = nr == 0 ? r : std::min(rate_min, r);
      nr++;
    }
  double grate = 0;
  int ng = 0;
  for (int x = 0; x < c->L; ++x)
    if (c->p_g2c[x] > 0) grate += c->p_g2c[x] / (4.0 * c->lay[x].n_pad), ng++;
  c->p_c2g_out.assign(c->L, 0.0);
  for (int x = 0; x < c->L; ++x) {
    const double fetch_b = late ? (double)c->cb : fbx(x);  // bytes per element the next fetch will move
    c->p_c2g_out[x] = (c->p_c2g[x] > 0 && fetch_b == fbx(x)) ? c->p_c2g[x]
                      : (nr ? (late ? rate_min : rate / nr) * fetch_b * c->lay[x].n_pad : 0.0);
    if (c->p_g2c[x] <= 0 && ng) c->p_g2c[x] = grate / ng * 4.0 * c->lay[x].n_pad;
    c->p_ocpu[x] = c->cpu_elems.load() > 0
                       ? c->cpu_ms.load() / c->n_threads / (double)c->cpu_elems.load() * c->lay[x].n_pad
                       : 0.0;
  }
  o->n_layers = c->L;
  o->t_fp = c->p_fp.data();
  o->t_bp = c->p_bp.data();
  o->t_c2g = c->p_c2g_out.data();
  o->t_g2c = c->p_g2c.data();
  o->t_stage = c->p_stage.data();
  o->t_opt_gpu = c->p_ogpu.data();
  o->t_opt_cpu = c->p_ocpu.data();
  o->t_async = c->n_async ? c->t_async_ms / c->n_async : 0.0;
  o->slot_bytes = c->p_slot_i.data();
  o->gstate_bytes = c->p_gstate_i.data();
  o->fixed_bytes = 0;
  size_t fr = 0, tot = 0;
  cudaMemGetInfo(&fr, &tot);
  // S_avail = what the engine holds now (ring + G states) + what is still free - margin
  int64_t held = c->ring_bytes_for(c->ring_alloc);
  for (int x = 0; x < c->L; ++x)
    if (c->g[x].master) held += 12 * c->lay[x].n_pad;
  o->s_avail = c->cfg.device_budget_bytes > 0 ? c->cfg.device_budget_bytes
                                              : held + (int64_t)fr - ((int64_t)2 << 30);
  o->duplex = (c->cfg.flags & SH_FLAG_DUPLEX) ? 1 : 0;
  o->cpu_hard = (c->cfg.flags & SH_FLAG_CPU_HARD) ? 1 : 0;
  o->cpu_util_max = c->cfg.cpu_util_max > 0.0 ? c->cfg.cpu_util_max : 0.85;
  // decoupling needs a landing buffer per host layer: otherwise the ring's grad halves are what
  // absorbs the D2H backlog when the CPU Adam is slower than BP (measured: a 7-slot ring with a
  // 4-deep landing ring stalled BP every 4 layers on the C4 model)
  // (with SH_FLAG_GROW_LANDING a private store grows its landing ring when the autotuner
  // decouples, see sh_autotune_window)
  // ... or, with SH_FLAG_FILL_GPU, a gradient pool sized for the backward backlog (R27): the pool and the
  // lowest-first offload order change the R22 finding, which was measured with slot-bound grad halves
  // and a FIFO queue (SH_DECOUPLE_ANY=1 forces decoupling for A/B runs)
  static const bool any = [] {
    const char* e = getenv("SH_DECOUPLE_ANY");
    return e && e[0] == '1';
  }();
  o->decouple = (c->cfg.flags & SH_FLAG_DECOUPLE) && !c->clip &&
                        (c->D >= c->L || (!c->shared && (c->cfg.flags & SH_FLAG_GROW_LANDING)) ||
                         (c->cfg.flags & SH_FLAG_FILL_GPU) || any) ? 1 : 0;
  o->landing_buffers = c->D;
  o->fp_serial = o->decouple;  // R23: a decoupled (short) ring must also cover the serialised fetch queue
  o->fill_gpu = o->decouple && (c->cfg.flags & SH_FLAG_FILL_GPU) ? 1 : 0;
  return SH_OK;
}

sh_status sh_set_window(sh_ctx* c, int32_t w) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  if (c->phase != sh_ctx::IDLE) {
    set_error("sh_set_window: only between steps");
    return SH_ERR_STATE;
  }
  if (w < 0 || w > c->L) {
    set_error("sh_set_window: window %d outside 0..%d", w, c->L);
    return SH_ERR_INVALID;
  }
  if (c->clip && c->D < c->L - w) {
    set_error("sh_set_window: clip mode needs a landing buffer per host layer");
    return SH_ERR_INVALID;
  }
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  if (w == c->w) return SH_OK;
  return apply_window(c, w);
}

sh_status sh_set_window_ring(sh_ctx* c, int32_t w, int32_t ring) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  if (ring < 0) {
    set_error("sh_set_window_ring: ring_slots must be >= 0");
    return SH_ERR_INVALID;
  }
  if (c->clip && ring > 0 && ring < w + 1) {
    set_error("sh_set_window_ring: clip mode pins the GPU-optimised layers' grads: ring must be >= window + 1");
    return SH_ERR_INVALID;
  }
  if (c->byte_ring() && ring > 0) {
    set_error("sh_set_window_ring: the ring is a fixed-byte buffer (ring_bytes); ring_slots must be 0");
    return SH_ERR_INVALID;
  }
  if (c->phase != sh_ctx::IDLE) {
    set_error("sh_set_window_ring: only between steps");
    return SH_ERR_STATE;
  }
  if (w < 0 || w > c->L) {
    set_error("sh_set_window_ring: window %d outside 0..%d", w, c->L);
    return SH_ERR_INVALID;
  }
  sh_status st = check_failed(c);
  if (st != SH_OK) return st;
  if (w == c->w && ring == c->ring_cap) return SH_OK;
  const int old_cap = c->ring_cap;
  c->ring_cap = ring;
  st = apply_window(c, w);
  if (st != SH_OK) {  // the window did not change: neither does the ring cap
    c->ring_cap = old_cap;
    c->n_active = std::min(c->ring_for(c->w), std::max(c->ring_alloc, 1));
    c->d = c->n_active - 1;
  }
  return st;
}

sh_status sh_autotune_window(sh_ctx* c, const sh_profile* ov, int32_t* wout) {
  clear_error();
  if (!c) return SH_ERR_INVALID;
  if (c->byte_ring()) {
    set_error("sh_autotune_window: a fixed-byte ring (ring_bytes) sets the window by bytes, not by the P1/P2 search");
    return SH_ERR_UNSUPPORTED;
  }
  sh_profile p{};
  if (ov) {
    p = *ov;
  } else {
    sh_status st = sh_get_profile(c, &p);
    if (st != SH_OK) return st;
  }
  sh_solve_report rep{};
  sh_status st = sh_solve_window(&p, &rep);
  if (st != SH_OK) return st;
  c->autotune_pending = false;
  if (getenv("SH_DEBUG_AUTOTUNE")) {
    double fp = 0, c2g = 0, g2c = 0, cpu = 0;
    for (int x = 0; x < p.n_layers; ++x)
      fp += p.t_fp[x], c2g += p.t_c2g ? p.t_c2g[x] : 0, g2c += p.t_g2c ? p.t_g2c[x] : 0,
          cpu += p.t_opt_cpu ? p.t_opt_cpu[x] : 0;
    const double n = p.n_layers;
    fprintf(stderr, "[sh autotune] w=%d ring=%d reason=%d decouple=%d fp_serial=%d fill=%d s_avail=%.1fGB "
            "mean t_fp=%.2f t_c2g=%.2f t_g2c=%.2f t_cpu=%.2f ms, slot=%.2fGB gstate=%.2fGB\n",
            rep.window, rep.ring_slots, rep.reason, p.decouple, p.fp_serial, p.fill_gpu, p.s_avail / 1e9, fp / n,
            c2g / n, g2c / n, cpu / n, p.slot_bytes ? p.slot_bytes[0] / 1e9 : 0.0,
            p.gstate_bytes ? p.gstate_bytes[0] / 1e9 : 0.0);
  }
  int32_t w = rep.window;
  int32_t ring = p.decouple && !c->clip ? rep.ring_slots : 0;
  if (c->shared) {  // one shared host store: the whole job must switch to the same window
    if (c->rank == 0) c->ctl->window.store((int64_t)w | ((int64_t)ring << 32));
    if (!shm_barrier(c, 4, "autotuned window agreement")) return check_failed(c);
    const int64_t v = c->ctl->window.load();
    w = (int32_t)(v & 0xffffffff);
    ring = (int32_t)(v >> 32);
    if (!shm_barrier(c, 5, "autotuned window read")) return check_failed(c);
  }
  // a decoupled ring needs a landing buffer per host-optimised layer (R22): with a private store
  // the landing ring grows into the host RAM the layers joining the GPU set give back -- if that
  // RAM (plus what is free now) cannot hold it, stay coupled
  const int64_t lb = align_up(4 * c->max_pad, 4096);
  const char* any_e = getenv("SH_DECOUPLE_ANY");
  // decouple on the gradient pool alone (no landing growth): forced, or a pool-sized ring (R27)
  const bool any = (any_e && any_e[0] == '1') || rep.reason == 3;
  if (ring > 0 && c->D < c->L - w && !any) {
    int64_t freed = 0;
    for (int x = c->w; x < w; ++x)
      if (c->hblocks[x].p && c->hblocks[x].fd < 0) freed += (int64_t)c->hblocks[x].bytes;
    const int64_t need = (int64_t)(c->L - w) * lb + (int64_t)(8ll << 30);  // + headroom
    if (c->shared || mem_available_bytes() + freed < need) ring = 0;
  }
  // apply; if HBM turns out short (the solver's S_avail is an estimate), step the window down
  const int w_old = c->w;
  st = sh_set_window_ring(c, w, ring);
  while (st == SH_ERR_OOM_DEVICE && w > w_old) {
    --w;
    if (ring > 0) ring = std::min(ring, w + 1);
    st = sh_set_window_ring(c, w, ring);
  }
  if (st == SH_ERR_OOM_DEVICE) st = sh_set_window_ring(c, w_old, 0);  // restore the warm-up window
  // one landing buffer per host layer: required by a decoupled ring; with SH_FLAG_GROW_LANDING also
  // for a coupled one (the D2H issuer then never waits for the CPU Adam to free a buffer)
  if (st == SH_OK && ((c->ring_cap > 0 && !any) || (c->cfg.flags & SH_FLAG_GROW_LANDING)) && c->D < c->L - c->w) {
    st = grow_landing(c, c->L - c->w);
    if (st != SH_OK) {  // host RAM after all too short: keep the short ring (coupled)
      clear_error();
      st = c->ring_cap > 0 ? sh_set_window_ring(c, c->w, 0) : SH_OK;
    }
  }
  if (st == SH_OK && (c->cfg.flags & SH_FLAG_LATE_SHADOW)) st = enable_late_shadow(c);
  if (wout) *wout = c->w;
  return st;
}

sh_status sh_read_layer(sh_ctx* c, int32_t layer, int32_t what, void* dst) {
  clear_error();
  if (!c || !dst) return SH_ERR_INVALID;
  if (layer < -1 || layer >= c->L || what < 0 || what > 4) {
    set_error("sh_read_layer: bad layer %d / what %d", layer, what);
    return SH_ERR_INVALID;
  }
  if (c->phase != sh_ctx::IDLE) {
    set_error("sh_read_layer: only between steps");
    return SH_ERR_STATE;
  }
  sh_status st = sync_all(c);
  if (st != SH_OK && !c->failed.load()) return st;
  const LayerLayout& Lx = layer < 0 ? c->res : c->lay[layer];
  const int64_t n = Lx.n_pad;
  if (layer >= 0 && !c->is_g(layer) && c->spilled[layer] && what != SH_READ_GRAD) {  // NEXT-2: from the file
    const int64_t rb = sp_rb(c, layer), fb = sp_file_bytes(c, layer);
    AlignedBuf t(fb);
    if (!t.p) return SH_ERR_OOM_HOST;
    st = spill_file_io(c, false, layer, t.p, fb);
    if (st != SH_OK) return st;
    if (what == SH_READ_COMPUTE) {
      if (c->bf16) {
        std::vector<uint16_t> b16(n);
        if (c->shadow) std::memcpy(b16.data(), t.b() + 3 * rb, 2 * n);
        else if (c->split) std::memcpy(b16.data(), t.b(), 2 * n);
        else cpu::cast_bf16_range(t.f(), b16.data(), 0, n);
        unpack_layer_u16(Lx, b16.data(), static_cast<uint16_t*>(dst));
      } else {
        unpack_layer(Lx, t.f(), static_cast<float*>(dst));
      }
      return SH_OK;
    }
    if (what == SH_READ_PARAM && c->split) {
      std::vector<float> mst(n);
      const uint16_t* h16 = reinterpret_cast<const uint16_t*>(t.b());
      join_par(c, h16, h16 + n, mst.data(), 0, n);
      unpack_layer(Lx, mst.data(), static_cast<float*>(dst));
      return SH_OK;
    }
    unpack_layer(Lx, reinterpret_cast<const float*>(t.b() + what * rb), static_cast<float*>(dst));
    return SH_OK;
  }
  if (what == SH_READ_COMPUTE) {
    std::vector<uint8_t> tmp((size_t)c->cb * n);
    if (layer < 0) {
      CKC(c, cudaMemcpy(tmp.data(), c->res_compute, tmp.size(), cudaMemcpyDeviceToHost));
    } else if (c->is_g(layer)) {
      if (c->layer_slot[layer] >= 0) {
        CKC(c, cudaMemcpy(tmp.data(), c->slot_param(c->layer_slot[layer]), tmp.size(), cudaMemcpyDeviceToHost));
      } else {  // outside the ring (decoupled ring): the copy K1 would stage, from the HBM master
        std::vector<float> mst(n);
        CKC(c, cudaMemcpy(mst.data(), c->g[layer].master, 4 * n, cudaMemcpyDeviceToHost));
        if (c->bf16)
          cpu::cast_bf16_range(mst.data(), reinterpret_cast<uint16_t*>(tmp.data()), 0, n);
        else
          std::memcpy(tmp.data(), mst.data(), 4 * n);
      }
    } else {
      if (c->h_shadow[layer])
        std::memcpy(tmp.data(), c->h_shadow[layer], tmp.size());
      else if (c->bf16)
        cpu::cast_bf16_range(c->h_master[layer], reinterpret_cast<uint16_t*>(tmp.data()), 0, n);
      else
        std::memcpy(tmp.data(), c->h_master[layer], tmp.size());
    }
    if (c->bf16)
      unpack_layer_u16(Lx, reinterpret_cast<uint16_t*>(tmp.data()), static_cast<uint16_t*>(dst));
    else
      unpack_layer(Lx, reinterpret_cast<float*>(tmp.data()), static_cast<float*>(dst));
    return SH_OK;
  }
  std::vector<float> tmp(n);
  if (what == SH_READ_GRAD) {  // gradients of the last completed step
    if (layer < 0) {
      CKC(c, cudaMemcpy(tmp.data(), c->res_grad, 4 * n, cudaMemcpyDeviceToHost));
    } else if (c->is_g(layer) && c->k2_layer) {
      const int b = c->layer_gbuf[layer];
      if (b < 0 || c->gbuf_owner[b] != layer) {
        set_error("sh_read_layer: grads of layer %d were overwritten (%d GPU-layer grad buffers)", layer,
                  (int)c->gbuf.size());
        return SH_ERR_STATE;
      }
      CKC(c, cudaMemcpy(tmp.data(), c->gbuf[b], 4 * n, cudaMemcpyDeviceToHost));
    } else if (c->is_g(layer)) {  // clip mode: the pool buffer its K2 read (until another layer takes it)
      const int b = c->layer_gb[layer];
      if (b < 0 || c->gb_owner[b] != -1 || c->gradfree_gen[b] <= 0) {
        set_error("sh_read_layer: grads of layer %d not available", layer);
        return SH_ERR_STATE;
      }
      CKC(c, cudaMemcpy(tmp.data(), c->slot_grad(b), 4 * n, cudaMemcpyDeviceToHost));
    } else {
      const int k = c->last_landing[layer];
      if (k < 0 || c->landing_owner[k] != layer) {
        set_error("sh_read_layer: grads of layer %d were overwritten in the landing ring (depth %d)", layer, c->D);
        return SH_ERR_STATE;
      }
      std::memcpy(tmp.data(), c->landing[k], 4 * n);
    }
    unpack_layer(Lx, tmp.data(), static_cast<float*>(dst));
    return SH_OK;
  }
  if (layer < 0 || c->is_g(layer)) {
    const float* src = layer < 0 ? (what == 0 ? c->res_master : what == 1 ? c->res_m : c->res_v)
                                 : (what == 0 ? c->g[layer].master : what == 1 ? c->g[layer].m : c->g[layer].v);
    CKC(c, cudaMemcpy(tmp.data(), src, 4 * n, cudaMemcpyDeviceToHost));
  } else if (what == SH_READ_PARAM && c->split) {
    join_par(c, c->h_shadow[layer], c->h_lo[layer], tmp.data(), 0, n);
  } else {
    const float* src = what == 0 ? c->h_master[layer] : what == 1 ? c->h_m[layer] : c->h_v[layer];
    std::memcpy(tmp.data(), src, 4 * n);
  }
  unpack_layer(Lx, tmp.data(), static_cast<float*>(dst));
  return SH_OK;
}

sh_status sh_stats(sh_ctx* c, sh_stats_t* o) {
  clear_error();
  if (!c || !o) return SH_ERR_INVALID;
  if (c->phase == sh_ctx::IDLE) sync_all(c);
  o->step = c->step;
  o->window = c->w;
  o->n_slots = c->ring_alloc;
  o->host_bytes = (int64_t)c->host_bytes;
  o->device_bytes = c->device_bytes;
  o->h2d_bytes = c->h2d_bytes.load();
  o->d2h_bytes = c->d2h_bytes.load();
  o->h2d_copies = c->h2d_copies.load();
  o->d2h_copies = c->d2h_copies.load();
  o->stage_launches = c->stage_launches.load();
  o->h2d_busy_ms = c->h2d_busy;
  o->d2h_busy_ms = c->d2h_busy;
  o->h2d_profiled_bytes = c->h2d_prof_bytes;
  o->d2h_profiled_bytes = c->d2h_prof_bytes;
  o->cpu_adam_ms = c->cpu_ms.load();
  o->cpu_adam_elems = c->cpu_elems.load();
  o->cpu_adam_shadow_elems = c->cpu_shadow_elems.load();
  o->spill_read_bytes = c->spill_rd_bytes.load();
  o->spill_write_bytes = c->spill_wr_bytes.load();
  o->spill_io_ms = c->spill_io_ms.load();
  o->spill_direct = c->spill_direct ? 1 : 0;
  o->spill_uring = c->n_spilled > 0 && spill::uring_available() ? 1 : 0;
  o->hybrid_layers = c->n_hyb;
  o->hybrid_updates = c->hyb_updates.load();
  o->hybrid_h2d_bytes = c->hyb_h2d.load();
  o->hybrid_d2h_bytes = c->hyb_d2h.load();
  {
    int n = 0;
    for (int x = c->w; x < c->L; ++x) n += c->h_shadow[x] != nullptr;
    o->shadow_layers = n;
  }
  o->cpu_wait_ms = c->cpu_wait_ms.load();
  o->k2_ms_last = c->k2_ms_last;
  o->k2_bytes_last = c->k2_bytes_last;
  o->k2_launches_last = c->k2_launches_last;
  o->cpu_threads = c->n_threads;
  o->profiled_steps = c->profiled_steps;
  o->k2_ms_sum = c->k2_ms_sum;
  o->k2_bytes_sum = c->k2_bytes_sum;
  o->k2_samples = c->k2_samples;
  o->k3_ms_sum = c->k3_ms_sum;
  o->k3_bytes_sum = c->k3_bytes_sum;
  o->k3_samples = c->k3_samples;
  o->h2d_overlap_frac = c->h2d_overlap;
  o->d2h_overlap_frac = c->d2h_overlap;
  o->last_step_ms = c->last_step_ms;
  o->compute_busy_ms = c->compute_busy_ms;
  o->ring_bytes = c->ring_bytes_for(c->ring_alloc);
  o->spill_bytes = (int64_t)c->spill_bytes;
  o->landing_buffers = c->D;
  o->spilled_layers = c->n_spilled;
  o->numa_nodes = c->numa_nodes;
  o->numa_policy = c->numa_policy;
  o->numa_gpu_node = c->numa_gpu;
  o->numa_pinned_workers = c->numa_pinned.load();
  o->numa_bound_bytes = c->numa_bound.load();
  return SH_OK;
}

sh_status sh_get_trace(sh_ctx* c, sh_trace_event* out, int32_t cap, int32_t* n_out) {
  clear_error();
  if (!c || !n_out) return SH_ERR_INVALID;
  if (c->phase == sh_ctx::IDLE) sync_all(c);
  *n_out = (int32_t)c->trace.size();
  for (int i = 0; i < (int)c->trace.size() && i < cap && out; ++i) out[i] = c->trace[i];
  return SH_OK;
}

sh_status sh_destroy(sh_ctx* c) {
  clear_error();
  if (!c) return SH_OK;
  if (!c->failed.load()) sync_all(c);
  {
    std::lock_guard<std::mutex> g(c->pmu);
    c->pool_stop = true;
  }
  c->pcv.notify_all();
  for (auto& t : c->workers) t.join();
  c->failed.store(1);  // release any issuer wait
  notify_state(c);
  c->ih2d.stop();
  c->id2h.stop();
  for (cudaStream_t s : {c->h2d, c->d2h, c->stage, c->comm, c->k3s, c->hyb_in, c->hyb_k, c->hyb_out})
    if (s) cudaStreamSynchronize(s);
  if (c->cs) cudaStreamSynchronize(c->cs);
  if (!c->nccl_aborted.load()) {  // an aborted communicator is already freed
    if (c->nccl_fetch) g_nccl.CommDestroy(c->nccl_fetch);
    if (c->nccl) g_nccl.CommDestroy(c->nccl);
  }
  if (c->partials_all) cudaFree(c->partials_all);
  if (c->fp32_stage) cudaFree(c->fp32_stage);
  for (char* p : c->hyb_stg) cudaFree(p);
  for (auto* v : {&c->ev_stg_in, &c->ev_stg_k2, &c->ev_stg_free})
    for (cudaEvent_t e : *v)
      if (e) cudaEventDestroy(e);
  if (c->hc_seg) {
    cudaHostUnregister(c->hc_seg);
    munmap(c->hc_seg, c->hc_bytes);
  }
  host_block_free(reinterpret_cast<char*>(c->hc_tmp), c->hc_bytes);
  for (int x = 0; x < c->L; ++x) free_g(c, x);
  for (float* p : c->gbuf) cudaFree(p);
  for (float* p : c->xgrad) cudaFree(p);
  for (float* p : c->xres) cudaFree(p);
  for (auto e : c->ev_gbuf_free) cudaEventDestroy(e);
  for (auto e : c->ev_gbuf_ready) cudaEventDestroy(e);
  if (c->ring) cudaFree(c->ring);
  if (c->res_master) cudaFree(c->res_master);
  if (c->partials) cudaFree(c->partials);
  for (auto* v : {&c->ev_param_free, &c->ev_grad_done, &c->ev_grad_free, &c->ev_reduced, &c->ev_k3_buf, &c->ev_arrive,
                  &c->ev_upd})
    for (auto e : *v)
      if (e) cudaEventDestroy(e);
  for (auto& P : c->prof) {
    for (auto* v : {&P.fp0, &P.fp1, &P.bp0, &P.bp1, &P.c2g0[0], &P.c2g1[0], &P.c2g0[1], &P.c2g1[1],
                    &P.g2c0, &P.g2c1, &P.st0, &P.st1, &P.k30, &P.k31, &P.k2l0, &P.k2l1})
      for (auto e : *v)
        if (e) cudaEventDestroy(e);
    if (P.k2a) cudaEventDestroy(P.k2a);
    if (P.t0) cudaEventDestroy(P.t0);
    if (P.k2b) cudaEventDestroy(P.k2b);
  }
  if (c->ev_cs_mark) cudaEventDestroy(c->ev_cs_mark);
  if (c->ev_comm_done) cudaEventDestroy(c->ev_comm_done);
  if (c->ev_k3_last) cudaEventDestroy(c->ev_k3_last);
  for (int i = 0; i < 2; ++i) {
    if (c->ev_res_k3[i]) cudaEventDestroy(c->ev_res_k3[i]);
    if (c->ev_norm[i]) cudaEventDestroy(c->ev_norm[i]);
  }
  for (cudaStream_t s : {c->h2d, c->d2h, c->stage, c->comm, c->k3s, c->hyb_in, c->hyb_k, c->hyb_out})
    if (s) cudaStreamDestroy(s);
  for (auto& b : c->hshadow) host_block_free(b.p, b.bytes);
  c->stg_cv.notify_all();
  c->spill_rd.stop();
  c->spill_wr.stop();
  for (char* p : c->stg_all) host_block_free(p, c->stg_bytes);
  for (auto& b : c->hblocks) {
    if (b.fd >= 0) {
      close(b.fd);
    } else {
      host_block_free(b.p, b.bytes);
    }
  }
  for (int k = 0; k < 2; ++k) {
    host_block_free(c->bounce[k], c->bounce_bytes);
    if (c->ev_bounce[k]) cudaEventDestroy(c->ev_bounce[k]);
  }
  if (c->ctl) munmap(c->ctl, c->ctl_bytes);
  host_block_free(c->hland.p, c->hland.bytes);
  delete c;
  return SH_OK;
}

sh_status sh_spill_probe(const char* dir, int64_t bytes, double* read_gbs, double* write_gbs, int32_t* direct) {
  clear_error();
  if (!dir || bytes <= 0 || !read_gbs || !write_gbs) return SH_ERR_INVALID;
  char path[4096];
  snprintf(path, sizeof(path), "%s/sh_spill_probe_%d.bin", dir, (int)getpid());
  int fd = open(path, O_RDWR | O_CREAT | O_EXCL | O_DIRECT, 0600);
  const int d = fd >= 0;
  if (fd < 0 && errno == EINVAL) fd = open(path, O_RDWR | O_CREAT | O_EXCL, 0600);
  if (fd < 0) {
    set_error("sh_spill_probe: open(%s): %s", path, strerror(errno));
    return SH_ERR_INVALID;
  }
  unlink(path);
  const size_t n = (size_t)align_up(bytes, 1 << 21);
  void* p = mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (p == MAP_FAILED || posix_fallocate(fd, 0, (off_t)n) != 0) {
    if (p != MAP_FAILED) munmap(p, n);
    close(fd);
    set_error("sh_spill_probe: no memory / disk space for %lld B", (long long)n);
    return SH_ERR_OOM_HOST;
  }
  std::memset(p, 0x5a, n);
  double t0 = now_ms();
  int r = spill::transfer(true, fd, p, n, 0);
  if (r == 0) fdatasync(fd);
  const double tw = now_ms() - t0;
  posix_fadvise(fd, 0, (off_t)n, POSIX_FADV_DONTNEED);
  t0 = now_ms();
  if (r == 0) r = spill::transfer(false, fd, p, n, 0);
  const double tr = now_ms() - t0;
  munmap(p, n);
  close(fd);
  if (r != 0) {
    set_error("sh_spill_probe: I/O failed: %s", strerror(-r));
    return SH_ERR_OOM_HOST;
  }
  *write_gbs = n / (tw / 1e3) / 1e9;
  *read_gbs = n / (tr / 1e3) / 1e9;
  if (direct) *direct = d;
  return SH_OK;
}

// ---- op-level entry points ------------------------------------------------------------
static bool ops_args_ok(int64_t n, int64_t n_decay, const void* const* ptrs, int np) {
  if (n < 0 || n % 8 != 0 || n_decay < 0 || n_decay > n || n_decay % 8 != 0) {
    set_error("op: n and n_decay must be multiples of 8 with 0 <= n_decay <= n");
    return false;
  }
  for (int i = 0; i < np; ++i)
    if (ptrs[i] && (reinterpret_cast<uintptr_t>(ptrs[i]) & 15)) {
      set_error("op: pointers must be 16-byte aligned");
      return false;
    }
  return true;
}

}  // extern "C"

namespace {
// Per-(device, stream) device scratch of the op entry points: K3's partials + completion ticket and
// K2's two dynamic-schedule counters.  Allocated and zeroed once (synchronously) on first use; every
// kernel leaves its part reset, so launches in stream order reuse it and launches on other streams or
// devices never share it.  Never freed (a few KB per stream handle).
struct OpScratch {
  double* k3 = nullptr;        // kSumsqMaxBlocks partials + ticket
  unsigned int* k2 = nullptr;  // 2 counters
};
OpScratch op_scratch(cudaStream_t st) {
  static std::mutex mu;
  static std::map<std::pair<int, cudaStream_t>, OpScratch> m;
  int dev = -1;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    cudaGetLastError();
    return {};
  }
  std::lock_guard<std::mutex> g(mu);
  auto it = m.find({dev, st});
  if (it != m.end()) return it->second;
  const size_t k3b = 8 * (kern::kSumsqMaxBlocks + 1);
  void* p = nullptr;
  if (cudaMalloc(&p, k3b + 64) != cudaSuccess || cudaMemset(p, 0, k3b + 64) != cudaSuccess) {
    cudaGetLastError();
    if (p) cudaFree(p);
    return {};
  }
  OpScratch o{static_cast<double*>(p), reinterpret_cast<unsigned int*>(static_cast<char*>(p) + k3b)};
  m[{dev, st}] = o;
  return o;
}
}  // namespace

extern "C" {

sh_status sh_op_adamw_gpu(float* p, float* m, float* v, const float* g, uint16_t* out16, float* out32,
                          int64_t n, int64_t n_decay, const sh_adam_scalars* sc, const float* coef,
                          void* stream) {
  clear_error();
  const void* ptrs[] = {p, m, v, g, out16, out32};
  if (!p || !m || !v || !g || !sc || (out16 && out32) || !ops_args_ok(n, n_decay, ptrs, 6))
    return SH_ERR_INVALID;
  kern::K2Args a{};
  a.sc = *sc;
  a.coef = coef;
  a.out_bf16 = out16 != nullptr;
  a.n_entries = 1;
  a.e[0] = kern::K2Entry{p, m, v, g, out16 ? (void*)out16 : (void*)out32, n, n_decay};
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (kern::k2_dynamic()) {
    a.sched = op_scratch(st).k2;
    if (!a.sched) {
      set_error("K2 schedule counters: allocation failed");
      return SH_ERR_OOM_DEVICE;
    }
  }
  const cudaError_t e = kern::adamw_multi(a, st);
  if (e != cudaSuccess) {
    set_error("K2 launch: %s", cudaGetErrorString(e));
    return SH_ERR_CUDA;
  }
  return SH_OK;
}

sh_status sh_op_adamw_cpu(float* p, float* m, float* v, const float* g, uint16_t* out16, int64_t n,
                          int64_t n_decay, const sh_adam_scalars* sc, int32_t use_coef, float coef,
                          int32_t n_threads) {
  clear_error();
  if (!p || !m || !v || !g || !sc || !ops_args_ok(n, n_decay, nullptr, 0)) return SH_ERR_INVALID;
  int T = n_threads > 0 ? n_threads : (int)std::thread::hardware_concurrency();
  if (T < 1) T = 1;
  const int64_t per = align_up(n / T + 1, 16);
  std::vector<std::thread> ts;
  for (int64_t b = 0; b < n; b += per) {
    const int64_t e = std::min(n, b + per);
    ts.emplace_back([=] { cpu::adamw_range(p, m, v, g, out16, b, e, n_decay, *sc, use_coef != 0, coef); });
  }
  for (auto& t : ts) t.join();
  return SH_OK;
}

sh_status sh_op_cast_bf16_gpu(const float* src, uint16_t* dst16, int64_t n, void* stream) {
  clear_error();
  const void* ptrs[] = {src, dst16};
  if (!src || !dst16 || !ops_args_ok(n, 0, ptrs, 2)) return SH_ERR_INVALID;
  const cudaError_t e = kern::cast_bf16(src, dst16, n, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) {
    set_error("K1 launch: %s", cudaGetErrorString(e));
    return SH_ERR_CUDA;
  }
  return SH_OK;
}

sh_status sh_op_cast_bf16_cpu(const float* src, uint16_t* dst16, int64_t n) {
  clear_error();
  if (!src || !dst16 || n < 0) return SH_ERR_INVALID;
  cpu::cast_bf16_range(src, dst16, 0, n);
  return SH_OK;
}

sh_status sh_op_master_split_cpu(const float* p, uint16_t* hi, uint16_t* lo, int64_t n) {
  clear_error();
  if (!p || !hi || !lo || n < 0) return SH_ERR_INVALID;
  cpu::split_range(p, hi, lo, 0, n);
  return SH_OK;
}

sh_status sh_op_master_join_cpu(const uint16_t* hi, const uint16_t* lo, float* p, int64_t n) {
  clear_error();
  if (!p || !hi || !lo || n < 0) return SH_ERR_INVALID;
  cpu::join_range(hi, lo, p, 0, n);
  return SH_OK;
}

sh_status sh_op_adamw_split_cpu(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t n,
                                int64_t n_decay, const sh_adam_scalars* sc, int32_t use_coef, float coef,
                                int32_t n_threads) {
  clear_error();
  if (!hi || !lo || !m || !v || !g || !sc || !ops_args_ok(n, n_decay, nullptr, 0)) return SH_ERR_INVALID;
  int T = n_threads > 0 ? n_threads : (int)std::thread::hardware_concurrency();
  if (T < 1) T = 1;
  const int64_t per = align_up(n / T + 1, 16);
  std::vector<std::thread> ts;
  for (int64_t b = 0; b < n; b += per) {
    const int64_t e = std::min(n, b + per);
    ts.emplace_back([=] { cpu::adamw_range_split(hi, lo, m, v, g, b, e, n_decay, *sc, use_coef != 0, coef); });
  }
  for (auto& t : ts) t.join();
  return SH_OK;
}

sh_status sh_op_adamw_split_gpu(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t n,
                                int64_t n_decay, const sh_adam_scalars* sc, void* stream) {
  clear_error();
  const void* ptrs[] = {hi, lo, m, v, g};
  if (!hi || !lo || !m || !v || !g || !sc || !ops_args_ok(n, n_decay, ptrs, 5)) return SH_ERR_INVALID;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  kern::K2SplitArgs a{};
  a.sc = *sc;
  a.hi = hi;
  a.lo = lo;
  a.m = m;
  a.v = v;
  a.g = g;
  a.n = n;
  a.n_decay = n_decay;
  a.sched = op_scratch(st).k2;
  if (!a.sched) {
    set_error("K2S schedule counters: allocation failed");
    return SH_ERR_OOM_DEVICE;
  }
  const cudaError_t e = kern::adamw_split(a, st);
  if (e != cudaSuccess) {
    set_error("K2S launch: %s", cudaGetErrorString(e));
    return SH_ERR_CUDA;
  }
  return SH_OK;
}

sh_status sh_op_exec_reduce_gpu(float* dst, const float* const* src, int32_t n_src, int64_t n, float inv_k,
                                void* stream) {
  clear_error();
  if (n_src < 0 || n_src >= kern::kMaxExecutors || (n_src > 0 && !src)) {
    set_error("sh_op_exec_reduce_gpu: n_src %d outside 0..%d", n_src, kern::kMaxExecutors - 1);
    return SH_ERR_INVALID;
  }
  kern::K4Args a{};
  a.dst = dst;
  a.n_src = n_src;
  for (int e = 0; e < n_src; ++e) a.src[e] = src[e];
  a.n = n;
  a.inv_k = inv_k;
  const void* ptrs[kern::kMaxExecutors + 1] = {dst};
  for (int e = 0; e < n_src; ++e) ptrs[e + 1] = src[e];
  if (!ops_args_ok(n, 0, ptrs, n_src + 1)) return SH_ERR_INVALID;
  const cudaError_t e = kern::exec_reduce(a, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) {
    set_error("sh_op_exec_reduce_gpu: %s", cudaGetErrorString(e));
    return SH_ERR_CUDA;
  }
  return SH_OK;
}

sh_status sh_op_sumsq_gpu(const float* g, int64_t n, double* out_dev, void* stream) {
  clear_error();
  const void* ptrs[] = {g};
  if (!g || !out_dev || !ops_args_ok(n, 0, ptrs, 1)) return SH_ERR_INVALID;
  // scratch (partials + completion ticket) private to this device and stream: concurrent calls on
  // other streams or devices never share it
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  double* scratch = op_scratch(st).k3;
  if (!scratch) {
    set_error("K3 scratch allocation failed");
    return SH_ERR_OOM_DEVICE;
  }
  const cudaError_t e = kern::sumsq(g, n, scratch, out_dev, st);
  if (e != cudaSuccess) {
    set_error("K3 launch: %s", cudaGetErrorString(e));
    return SH_ERR_CUDA;
  }
  return SH_OK;
}

}  // extern "C"
