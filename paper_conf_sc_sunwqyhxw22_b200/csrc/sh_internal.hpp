// Internal declarations shared by the engine translation units (not part of the ABI).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "sh.h"

namespace sh {

// ---- errors -----------------------------------------------------------------------
void set_error(const char* fmt, ...) __attribute__((format(printf, 1, 2)));
void clear_error();

// ---- layout -------------------------------------------------------
// Each tensor is padded to kPad elements (512 B of fp32, 256 B of bf16) so every tensor
// starts 256-B aligned in every slot (fixed cuBLAS alignment class => same kernels for
// every window) and K1/K2/K3 can use 128-bit accesses with no tail.  Tensors with weight
// decay are placed first, so one split point n_decay describes the whole layer.
constexpr int64_t kPad = 128;

struct LayerLayout {
  int n_tensors = 0;
  std::vector<int64_t> numel;   // caller order
  std::vector<uint8_t> wd;      // caller order
  std::vector<int64_t> offset;  // caller tensor k -> element offset inside the padded layer
  int64_t n_raw = 0;            // Σ numel
  int64_t n_pad = 0;            // padded total (multiple of kPad)
  int64_t n_decay = 0;          // [0, n_decay) decayed
};

bool make_layout(const sh_layer_shape& s, LayerLayout* out);
void pack_layer(const LayerLayout& L, const float* src, float* dst);    // caller order -> padded
void unpack_layer(const LayerLayout& L, const float* src, float* dst);  // padded -> caller order
void unpack_layer_u16(const LayerLayout& L, const uint16_t* src, uint16_t* dst);

// ---- kernels (kernels.cu) -----------------------------------------------------------
namespace spill {
constexpr size_t kAlign = 4096;  // O_DIRECT granularity (buffer address, length and file offset)
// true if this thread can use io_uring (else transfer() falls back to pread / pwrite)
bool uring_available();
// Blocking O_DIRECT transfer of bytes (multiple of kAlign) between buf (kAlign-aligned, ideally page-locked)
// and file offset off of fd (opened O_DIRECT).  0 or -errno.
int transfer(bool write, int fd, void* buf, size_t bytes, int64_t off);
}  // namespace spill

namespace kern {
struct K2Entry {
  float* p;
  float* m;
  float* v;
  const float* g;
  void* out;        // bf16 (uint16) or fp32 compute copy; may be null
  int64_t n;        // multiple of 8
  int64_t n_decay;  // multiple of 8
};
constexpr int kK2MaxEntries = 40;
struct K2Args {
  sh_adam_scalars sc;
  const float* coef;  // null: no clipping
  // null: static grid-stride schedule; else 2 zeroed device counters owned by the caller for this
  // stream (dynamic item distribution; the kernel leaves them zeroed); never shared by launches that
  // may run concurrently
  unsigned int* sched;
  int n_entries;
  int out_bf16;
  K2Entry e[kK2MaxEntries];
  int64_t item_start[kK2MaxEntries + 1];
};
// true unless SH_K2_SCHED=static: K2 launches that carry counters use the dynamic item schedule
bool k2_dynamic();
// Launch K2 over args (item_start filled by the callee).  Returns the grid used.
cudaError_t adamw_multi(K2Args& a, cudaStream_t st, int* grid_out = nullptr);
// K2S: AdamW on a split master (hi = bf16 compute copy, lo = low 16 bits; m, v fp32), updated in place;
// bitwise the CPU pool's split AdamW.  No clipping.  sched: 2 zeroed device counters owned by the caller
// for this stream (left zeroed).  n, n_decay multiples of 8; pointers 16-byte aligned.
struct K2SplitArgs {
  sh_adam_scalars sc;
  uint16_t* hi;
  uint16_t* lo;
  float* m;
  float* v;
  const float* g;
  int64_t n;
  int64_t n_decay;
  unsigned int* sched;
};
cudaError_t adamw_split(const K2SplitArgs& a, cudaStream_t st);
cudaError_t cast_bf16(const float* src, uint16_t* dst, int64_t n, cudaStream_t st);
constexpr int kSumsqMaxBlocks = 1184;  // 148 SMs x 8
// Deterministic Σ g^2 in fp64 -> *out (device).  scratch: kSumsqMaxBlocks + 1 doubles, zeroed
// once (the last word is the block ticket, reset by the kernel); one scratch per stream.
cudaError_t sumsq(const float* g, int64_t n, double* scratch, double* out, cudaStream_t st);
// norm = sqrt(Σ partials[0..n)) in index order; coef = min(1, max_norm/(norm+1e-6)) (fp32)
cudaError_t norm_finalize(const double* partials, int n, double max_norm, double* norm_out,
                          float* coef_out, cudaStream_t st);
// K4 (NEXT-3 executors): dst = ((dst + src[0]) + src[1] + ...) * inv_k elementwise (n multiple of 8).
constexpr int kMaxExecutors = 8;
struct K4Args {
  float* dst;
  const float* src[kMaxExecutors];
  int n_src;
  int64_t n;
  float inv_k;
};
cudaError_t exec_reduce(const K4Args& a, cudaStream_t st);
// Data parallel with reduce-scattered host layers: out[x] = all[0][x] for x < w_g (GPU-optimised
// layers, full gradients on every rank) and x = n-1 (resident set); out[x] = sum_r all[r][x] in
// rank order for the host layers (each rank holds the sum of squares of its slice).
cudaError_t fold_partials(const double* all, int world, int n, int w_g, double* out, cudaStream_t st);
int sm_count();
int64_t launches();
}  // namespace kern

// ---- CPU Adam (cpu_adam.cpp) ----------------------------------------------------------
namespace cpu {
// Elements [begin, end) of one padded layer (begin/end multiples of 16 or end == n).
void adamw_range(float* p, float* m, float* v, const float* g, uint16_t* out16, int64_t begin,
                 int64_t end, int64_t n_decay, const sh_adam_scalars& sc, bool use_coef,
                 float coef);
void cast_bf16_range(const float* src, uint16_t* dst, int64_t begin, int64_t end);
uint16_t rna_bf16(float x);
// Split master (R25): hi = rna_bf16(p), lo = low 16 bits of p; p = (hi << 16) + sext16(lo).
void adamw_range_split(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t begin, int64_t end,
                       int64_t n_decay, const sh_adam_scalars& sc, bool use_coef, float coef);
void split_range(const float* src, uint16_t* hi, uint16_t* lo, int64_t begin, int64_t end);
void join_range(const uint16_t* hi, const uint16_t* lo, float* dst, int64_t begin, int64_t end);
bool has_avx512();
}  // namespace cpu

// ---- NUMA placement (numa.cpp) ---------------------------------------------------------
namespace numa {
constexpr int kNone = -1;        // no binding / not pinned
constexpr int kInterleave = -2;  // page-interleaved over all nodes
struct Topology {
  std::vector<int> node_ids;          // online node ids (index = "node index")
  std::vector<std::vector<int>> cpus; // CPUs of each node
};
bool parse_cpulist(const char* s, std::vector<int>* out);
const Topology& topology();
int gpu_node_index(int device);
int resolve_policy(int policy, int n_nodes, bool shared);
int plan_node(int policy, int unit, int n_nodes, int gpu_node);
int worker_node(int policy, int tid, int n_threads, int gpu_node);
bool bind_range(void* p, size_t bytes, int node_index);
int node_of_page(const void* p);
bool pin_thread(int node_index);
}  // namespace numa

}  // namespace sh
