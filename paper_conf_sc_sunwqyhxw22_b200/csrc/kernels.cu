// Hot-path kernels of the offload engine for sm_100a.
//
//  K1 cast_bf16    fp32 master -> bf16 slot copy (restage of GPU-optimised layers in BP and
//                  the bf16 compute copy; PAPER.md:205 keeps the first window on the GPU).
//                  HBM-bound: 6 B/element.
//  K2 adamw_multi  fused multi-tensor AdamW over the GPU-optimised set (layers [0,w) and the
//                  resident embedding / positions / final LN), writing the
//                  new compute copy in place.  HBM-bound: 30 B/element (bf16 mode).
//  K3 sumsq        per-layer Σg² in fp64 with a fixed reduction tree (grad-norm for clipping;
//                  deterministic, no float atomics).  HBM-bound: 4 B/element.
//  K4 exec_reduce  the in-GPU all-reduce of the multi-stream executors (NEXT-3, PAPER.md:236-240:
//                  "an all-reduce operation to synchronize the gradients among parallel training
//                  workers before performing parameter updates"): g0 = (((g0+g1)+g2)+...)*inv_k
//                  in a fixed order.  HBM-bound: 4(k+1) B/element.
//
// None of these is a contraction, so there is no tensor-core work here: the rules that matter
// are 128-bit coalesced accesses, enough bytes in flight per SM, and a grid sized in
// multiples of the 148 SMs (persistent blocks striding over work items).
//
// Numerics: every floating-point op is an explicit
// round-to-nearest intrinsic so the compiler can neither contract nor reassociate, and the
// CPU AdamW (cpu_adam.cpp) executes the identical sequence => bitwise-identical results for
// any split of layers between GPU and CPU, i.e. for every window size.
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "sh_internal.hpp"

namespace sh {
namespace kern {

namespace {

// bf16 rounding of every compute copy: round to nearest, ties away from zero (RNA, R25) --
// the rounding under which the host store's split master (hi = the compute copy, lo = the low 16
// bits) is lossless; identical to cpu::rna_bf16.
__device__ __forceinline__ uint32_t rna_bf16_bits(float x) {
  uint32_t u = __float_as_uint(x);
  if ((u & 0x7fffffffu) > 0x7f800000u) return 0x7fc0u;  // canonical quiet NaN
  return (u + 0x8000u) >> 16;
}

__device__ __forceinline__ float4 ld_stream(const float* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ float4 ld_rw(const float* p) {
  return *reinterpret_cast<const float4*>(p);
}
__device__ __forceinline__ void st_f4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }

struct AdamS {
  float b1, b2, omb1, omb2, eps, nss, sqrt_bc2, decay;
};

__device__ __forceinline__ void adam_elem(float& p, float& m, float& v, float g, const AdamS& s,
                                          bool wd, bool use_coef, float coef) {
  if (use_coef) g = __fmul_rn(g, coef);
  m = __fmaf_rn(s.b1, m, __fmul_rn(s.omb1, g));
  v = __fmaf_rn(s.b2, v, __fmul_rn(s.omb2, __fmul_rn(g, g)));
  const float d = __fadd_rn(__fdiv_rn(__fsqrt_rn(v), s.sqrt_bc2), s.eps);
  const float pp = wd ? __fmul_rn(p, s.decay) : p;
  p = __fmaf_rn(s.nss, __fdiv_rn(m, d), pp);
}

// K2: one work item = 1024*U consecutive elements of one entry.  Thread t of the block handles
// elements base + u*1024 + 4t .. +3 for u in [0, U): every float4 load/store of a warp touches 512
// contiguous bytes; 4U independent 16-B loads in flight per thread (U = 4 by default, tuned on
// B200 with tools/bench_kernels.py).
//
// kDyn: dynamic work distribution.  Instead of the static grid stride, each block takes its next
// item from a global counter (a.sched[0], one atomicAdd per 4096-element item, broadcast through
// shared memory).  Under concurrency -- a K3 / K1 / GEMM on another stream holding some SMs when K2
// starts, copy-engine traffic -- blocks that start late simply take fewer items instead of
// leaving a tail of statically assigned work.  Items still arrive in increasing order per block,
// so the entry cursor stays monotone.  The last block to finish (a.sched[1] ticket) resets both
// counters for the next launch on the same stream.  Same per-element arithmetic => bitwise
// identical to the static kernel.
template <bool kBf16Out, int U, int kMinBlocks = 0, bool kDyn = false>
__global__ void __launch_bounds__(256, kMinBlocks) k2_adamw_kernel(const __grid_constant__ K2Args a) {
  const AdamS s{a.sc.beta1, a.sc.beta2, a.sc.omb1, a.sc.omb2, a.sc.eps, -a.sc.step_size,
                a.sc.sqrt_bc2, a.sc.decay};
  const bool use_coef = a.coef != nullptr;
  const float coef = use_coef ? *a.coef : 1.0f;
  const int64_t n_items = a.item_start[a.n_entries];
  int e = 0;
  __shared__ unsigned int s_item[2];
  int64_t item;
  int parity = 0;
  auto grab = [&]() -> int64_t {
    if (threadIdx.x == 0) s_item[parity] = atomicAdd(a.sched, 1u);
    __syncthreads();  // s_item[parity ^ 1] is free again: every thread read it before this barrier
    const int64_t it = s_item[parity];
    parity ^= 1;
    return it;
  };
  if constexpr (kDyn) item = grab();
  else item = blockIdx.x;
  for (; item < n_items; item = kDyn ? grab() : item + gridDim.x) {
    while (item >= a.item_start[e + 1]) ++e;  // items are visited in increasing order
    const K2Entry& E = a.e[e];
    const int64_t base = (item - a.item_start[e]) * (1024 * U);
    float4 p[U], m[U], v[U], g[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u * 1024 + 4 * threadIdx.x;
      if (i < E.n) {
        p[u] = ld_rw(E.p + i);
        m[u] = ld_rw(E.m + i);
        v[u] = ld_rw(E.v + i);
        g[u] = ld_stream(E.g + i);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u * 1024 + 4 * threadIdx.x;
      if (i >= E.n) continue;
      const bool wd = i < E.n_decay;  // n_decay is a multiple of 8: uniform per float4
      adam_elem(p[u].x, m[u].x, v[u].x, g[u].x, s, wd, use_coef, coef);
      adam_elem(p[u].y, m[u].y, v[u].y, g[u].y, s, wd, use_coef, coef);
      adam_elem(p[u].z, m[u].z, v[u].z, g[u].z, s, wd, use_coef, coef);
      adam_elem(p[u].w, m[u].w, v[u].w, g[u].w, s, wd, use_coef, coef);
      st_f4(E.p + i, p[u]);
      st_f4(E.m + i, m[u]);
      st_f4(E.v + i, v[u]);
      if (E.out != nullptr) {
        if constexpr (kBf16Out) {
          uint2 o;
          o.x = rna_bf16_bits(p[u].x) | (rna_bf16_bits(p[u].y) << 16);
          o.y = rna_bf16_bits(p[u].z) | (rna_bf16_bits(p[u].w) << 16);
          *reinterpret_cast<uint2*>(static_cast<uint16_t*>(E.out) + i) = o;
        } else {
          st_f4(static_cast<float*>(E.out) + i, p[u]);
        }
      }
    }
  }
  if constexpr (kDyn) {
    if (threadIdx.x == 0) {
      __threadfence();
      if (atomicAdd(a.sched + 1, 1u) == gridDim.x - 1) {  // every block has made its last grab
        a.sched[0] = 0;
        a.sched[1] = 0;
        __threadfence();
      }
    }
  }
}

// K2S: K2 on a host layer's SPLIT master (R25 / R28 "hybrid update"): the fp32 master is
// held as hi = rna_bf16(p) (the bf16 compute copy, here the layer's ring slot, updated in place) and
// lo = the low 16 bits of p (staged in HBM with m and v).  Per element: p = bits((hi << 16) + sext(lo)),
// the same adam_elem as K2, then hi' = rna_bf16(p), lo' = low 16 bits of p' -- exactly the CPU pool's
// split AdamW (cpu_adam.cpp adam_split_*), so a layer updated here or on the CPU ends bit-identical.
// HBM-bound: r hi 2 + lo 2 + m 4 + v 4 + g 4, w hi 2 + lo 2 + m 4 + v 4 = 28 B/element.  Same dynamic
// item schedule as K2 (one 4096-element item per block grab).
__global__ void __launch_bounds__(256, 3) k2_split_kernel(const __grid_constant__ K2SplitArgs a) {
  const AdamS s{a.sc.beta1, a.sc.beta2, a.sc.omb1, a.sc.omb2, a.sc.eps, -a.sc.step_size,
                a.sc.sqrt_bc2, a.sc.decay};
  constexpr int U = 4;
  const int64_t n_items = (a.n + 1024 * U - 1) / (1024 * U);
  __shared__ unsigned int s_item[2];
  int parity = 0;
  for (;;) {
    if (threadIdx.x == 0) s_item[parity] = atomicAdd(a.sched, 1u);
    __syncthreads();
    const int64_t item = s_item[parity];
    parity ^= 1;
    if (item >= n_items) break;
    const int64_t base = item * (1024 * U);
    float4 p[U], m[U], v[U], g[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u * 1024 + 4 * threadIdx.x;
      if (i < a.n) {
        const uint2 h = *reinterpret_cast<const uint2*>(a.hi + i);
        const uint2 l = *reinterpret_cast<const uint2*>(a.lo + i);
        auto join = [](uint32_t hh, uint32_t ll) {
          return __uint_as_float((hh << 16) + (uint32_t)(int32_t)(int16_t)(uint16_t)ll);
        };
        p[u] = make_float4(join(h.x & 0xffffu, l.x & 0xffffu), join(h.x >> 16, l.x >> 16),
                           join(h.y & 0xffffu, l.y & 0xffffu), join(h.y >> 16, l.y >> 16));
        m[u] = ld_rw(a.m + i);
        v[u] = ld_rw(a.v + i);
        g[u] = ld_stream(a.g + i);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u * 1024 + 4 * threadIdx.x;
      if (i >= a.n) continue;
      const bool wd = i < a.n_decay;  // n_decay is a multiple of 8: uniform per float4
      adam_elem(p[u].x, m[u].x, v[u].x, g[u].x, s, wd, false, 1.0f);
      adam_elem(p[u].y, m[u].y, v[u].y, g[u].y, s, wd, false, 1.0f);
      adam_elem(p[u].z, m[u].z, v[u].z, g[u].z, s, wd, false, 1.0f);
      adam_elem(p[u].w, m[u].w, v[u].w, g[u].w, s, wd, false, 1.0f);
      st_f4(a.m + i, m[u]);
      st_f4(a.v + i, v[u]);
      uint2 h, l;
      h.x = rna_bf16_bits(p[u].x) | (rna_bf16_bits(p[u].y) << 16);
      h.y = rna_bf16_bits(p[u].z) | (rna_bf16_bits(p[u].w) << 16);
      l.x = (__float_as_uint(p[u].x) & 0xffffu) | (__float_as_uint(p[u].y) << 16);
      l.y = (__float_as_uint(p[u].z) & 0xffffu) | (__float_as_uint(p[u].w) << 16);
      *reinterpret_cast<uint2*>(a.hi + i) = h;
      *reinterpret_cast<uint2*>(a.lo + i) = l;
    }
  }
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(a.sched + 1, 1u) == gridDim.x - 1) {  // every block has made its last grab
      a.sched[0] = 0;
      a.sched[1] = 0;
      __threadfence();
    }
  }
}

// K2, bulk-copy pipeline variant (SH_K2_IMPL=bulk).  The register-staged kernel above loads a work
// item, then computes and stores it: while a block is in its compute/store phase its loads are
// idle, and at 83 registers only 2 blocks fit per SM.  Here one 512-thread block per SM keeps the
// loads continuously in flight with the Blackwell bulk-copy engine: thread 0 streams the p, m, v
// and g slices of the next kBulkStages work items (4096 elements, 4 x 16 KB) into a ring of shared
// memory stages with cp.async.bulk, each stage completing a transaction-count mbarrier; all
// threads wait on the stage's barrier, run the same adam_elem on their 8 elements (conflict-free
// 16-B shared loads) and store the results to global memory straight from registers; after a
// block barrier thread 0 refills the stage with the item kBulkStages ahead.  Same per-element
// arithmetic as the other kernel => bitwise identical.
constexpr int kBulkThreads = 512;
constexpr int kBulkStages = 3;
template <int kItem>
constexpr size_t bulk_smem() { return (size_t)kBulkStages * 4 * kItem * sizeof(float) + 64; }

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra DONE;\n"
      "bra LAB_WAIT;\n"
      "DONE:\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_addr(dst)),
               "l"(src), "r"(bytes), "r"(smem_addr(bar))
               : "memory");
}
__device__ __forceinline__ float4 lds_f4(const float* p) { return *reinterpret_cast<const float4*>(p); }

template <bool kBf16Out, int kBulkItem, int kMinBlocks>
__global__ void __launch_bounds__(kBulkThreads, kMinBlocks) k2_adamw_bulk_kernel(const __grid_constant__ K2Args a) {
  constexpr int kU = kBulkItem / (4 * kBulkThreads);  // float4 per thread per array
  extern __shared__ __align__(128) unsigned char k2_smem[];
  float* stage_buf = reinterpret_cast<float*>(k2_smem);  // [kBulkStages][4 arrays][kBulkItem]
  uint64_t* bar = reinterpret_cast<uint64_t*>(k2_smem + (size_t)kBulkStages * 4 * kBulkItem * sizeof(float));
  const AdamS s{a.sc.beta1, a.sc.beta2, a.sc.omb1, a.sc.omb2, a.sc.eps, -a.sc.step_size,
                a.sc.sqrt_bc2, a.sc.decay};
  const bool use_coef = a.coef != nullptr;
  const float coef = use_coef ? *a.coef : 1.0f;
  const int64_t n_items = a.item_start[a.n_entries];
  if (threadIdx.x == 0) {
    for (int k = 0; k < kBulkStages; ++k) mbar_init(&bar[k], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  int e_prod = 0;  // producer's entry cursor (runs kBulkStages items ahead of the consumers)
  auto issue = [&](int64_t item, int stage) {
    while (item >= a.item_start[e_prod + 1]) ++e_prod;
    const K2Entry& E = a.e[e_prod];
    const int64_t base = (item - a.item_start[e_prod]) * kBulkItem;
    const int64_t cnt = E.n - base < kBulkItem ? E.n - base : kBulkItem;  // multiple of 8 elements
    const uint32_t bytes = (uint32_t)(cnt * sizeof(float));
    float* d = stage_buf + (size_t)stage * 4 * kBulkItem;
    mbar_expect_tx(&bar[stage], 4 * bytes);
    bulk_g2s(d, E.p + base, bytes, &bar[stage]);
    bulk_g2s(d + kBulkItem, E.m + base, bytes, &bar[stage]);
    bulk_g2s(d + 2 * kBulkItem, E.v + base, bytes, &bar[stage]);
    bulk_g2s(d + 3 * kBulkItem, E.g + base, bytes, &bar[stage]);
  };
  if (threadIdx.x == 0)
    for (int k = 0; k < kBulkStages; ++k) {
      const int64_t item = blockIdx.x + (int64_t)k * gridDim.x;
      if (item < n_items) issue(item, k);
    }
  int e = 0;
  int j = 0;
  for (int64_t item = blockIdx.x; item < n_items; item += gridDim.x, ++j) {
    const int stage = j % kBulkStages;
    while (item >= a.item_start[e + 1]) ++e;
    const K2Entry& E = a.e[e];
    const int64_t base = (item - a.item_start[e]) * kBulkItem;
    mbar_wait(&bar[stage], (uint32_t)((j / kBulkStages) & 1));
    const float* sp = stage_buf + (size_t)stage * 4 * kBulkItem;
    float4 p[kU], m[kU], v[kU], g[kU];
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int o = u * 4 * kBulkThreads + 4 * threadIdx.x;
      p[u] = lds_f4(sp + o);
      m[u] = lds_f4(sp + kBulkItem + o);
      v[u] = lds_f4(sp + 2 * kBulkItem + o);
      g[u] = lds_f4(sp + 3 * kBulkItem + o);
    }
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int64_t i = base + u * 4 * kBulkThreads + 4 * threadIdx.x;
      if (i >= E.n) continue;
      const bool wd = i < E.n_decay;  // n_decay is a multiple of 8: uniform per float4
      adam_elem(p[u].x, m[u].x, v[u].x, g[u].x, s, wd, use_coef, coef);
      adam_elem(p[u].y, m[u].y, v[u].y, g[u].y, s, wd, use_coef, coef);
      adam_elem(p[u].z, m[u].z, v[u].z, g[u].z, s, wd, use_coef, coef);
      adam_elem(p[u].w, m[u].w, v[u].w, g[u].w, s, wd, use_coef, coef);
      st_f4(E.p + i, p[u]);
      st_f4(E.m + i, m[u]);
      st_f4(E.v + i, v[u]);
      if (E.out != nullptr) {
        if constexpr (kBf16Out) {
          uint2 o;
          o.x = rna_bf16_bits(p[u].x) | (rna_bf16_bits(p[u].y) << 16);
          o.y = rna_bf16_bits(p[u].z) | (rna_bf16_bits(p[u].w) << 16);
          *reinterpret_cast<uint2*>(static_cast<uint16_t*>(E.out) + i) = o;
        } else {
          st_f4(static_cast<float*>(E.out) + i, p[u]);
        }
      }
    }
    __syncthreads();  // every thread is done reading this stage
    if (threadIdx.x == 0) {
      const int64_t nx = item + (int64_t)kBulkStages * gridDim.x;
      if (nx < n_items) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic reads before async writes
        issue(nx, stage);
      }
    }
  }
}

// K1: 8 elements per thread per iteration: 2 x 16-B loads -> 1 x 16-B store.
__global__ void __launch_bounds__(256) k1_cast_kernel(const float* __restrict__ src,
                                                     uint16_t* __restrict__ dst, int64_t n8) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n8;
       j += (int64_t)gridDim.x * blockDim.x) {
    const float4 a = ld_stream(src + 8 * j);
    const float4 b = ld_stream(src + 8 * j + 4);
    uint4 o;
    o.x = rna_bf16_bits(a.x) | (rna_bf16_bits(a.y) << 16);
    o.y = rna_bf16_bits(a.z) | (rna_bf16_bits(a.w) << 16);
    o.z = rna_bf16_bits(b.x) | (rna_bf16_bits(b.y) << 16);
    o.w = rna_bf16_bits(b.z) | (rna_bf16_bits(b.w) << 16);
    *reinterpret_cast<uint4*>(dst + 8 * j) = o;
  }
}

__device__ __forceinline__ double warp_sum(double x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

// Block-level fixed-tree sum of a per-thread double (blockDim == 256).
__device__ __forceinline__ double block_sum256(double x) {
  __shared__ double ws[8];
  x = warp_sum(x);
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = x;
  __syncthreads();
  double r = 0.0;
  if (threadIdx.x < 32) {
    r = threadIdx.x < 8 ? ws[threadIdx.x] : 0.0;
    r = warp_sum(r);
  }
  return r;  // valid in thread 0
}

// K3: one launch.  Block b sums float4 groups b*256+t, b*256+t+stride, ... (4 independent loads
// in flight per thread), reduces with a fixed warp-shuffle tree, writes partial[b]; the last block
// to finish (atomic ticket) sums partial[0..grid) in index order and resets the ticket.  The grid
// depends only on n, so the reduction tree -- and the result bits -- are fixed.
__global__ void __launch_bounds__(256) k3_sumsq_kernel(const float* __restrict__ g, int64_t n4,
                                                      double* __restrict__ partial,
                                                      unsigned int* __restrict__ ticket,
                                                      double* __restrict__ out) {
  const int64_t stride = (int64_t)gridDim.x * 256;
  int64_t j = blockIdx.x * 256ll + threadIdx.x;
  double acc0 = 0.0, acc1 = 0.0;
  for (; j + 3 * stride < n4; j += 4 * stride) {
    const float4 a = ld_stream(g + 4 * j);
    const float4 b = ld_stream(g + 4 * (j + stride));
    const float4 c = ld_stream(g + 4 * (j + 2 * stride));
    const float4 d = ld_stream(g + 4 * (j + 3 * stride));
    acc0 = fma((double)a.x, (double)a.x, acc0); acc1 = fma((double)a.y, (double)a.y, acc1);
    acc0 = fma((double)a.z, (double)a.z, acc0); acc1 = fma((double)a.w, (double)a.w, acc1);
    acc0 = fma((double)b.x, (double)b.x, acc0); acc1 = fma((double)b.y, (double)b.y, acc1);
    acc0 = fma((double)b.z, (double)b.z, acc0); acc1 = fma((double)b.w, (double)b.w, acc1);
    acc0 = fma((double)c.x, (double)c.x, acc0); acc1 = fma((double)c.y, (double)c.y, acc1);
    acc0 = fma((double)c.z, (double)c.z, acc0); acc1 = fma((double)c.w, (double)c.w, acc1);
    acc0 = fma((double)d.x, (double)d.x, acc0); acc1 = fma((double)d.y, (double)d.y, acc1);
    acc0 = fma((double)d.z, (double)d.z, acc0); acc1 = fma((double)d.w, (double)d.w, acc1);
  }
  for (; j < n4; j += stride) {
    const float4 a = ld_stream(g + 4 * j);
    acc0 = fma((double)a.x, (double)a.x, acc0); acc1 = fma((double)a.y, (double)a.y, acc1);
    acc0 = fma((double)a.z, (double)a.z, acc0); acc1 = fma((double)a.w, (double)a.w, acc1);
  }
  const double s = block_sum256(acc0 + acc1);
  __shared__ bool last;
  if (threadIdx.x == 0) {
    partial[blockIdx.x] = s;
    __threadfence();
    last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  double t = 0.0;
  for (int i = threadIdx.x; i < (int)gridDim.x; i += 256) t += __ldcg(partial + i);
  const double tot = block_sum256(t);
  if (threadIdx.x == 0) {
    *out = tot;
    *ticket = 0u;  // ready for the next launch on this scratch
  }
}

// K4: a block handles tiles of 4096 floats; thread t of the block owns the float4s at t*4 + 1024u
// (u < 4) of a tile, so every warp access is 512 contiguous bytes and all 4(n_src+1) 16-B loads of
// an iteration are in flight before the adds.  Executor buffers are streamed (L1 no-allocate), the
// destination is read and written in place.  The < 4096-float tail is done one float4 per thread.
__global__ void __launch_bounds__(256) k4_exec_reduce_kernel(const __grid_constant__ K4Args a) {
  const float f = a.inv_k;
  const int64_t tiles = a.n / 4096;
  for (int64_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const int64_t base = tile * 4096 + 4 * threadIdx.x;
    float4 x[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) x[u] = ld_rw(a.dst + base + 1024 * u);
    for (int s = 0; s < a.n_src; ++s) {
      float4 y[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) y[u] = ld_stream(a.src[s] + base + 1024 * u);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        x[u].x = __fadd_rn(x[u].x, y[u].x); x[u].y = __fadd_rn(x[u].y, y[u].y);
        x[u].z = __fadd_rn(x[u].z, y[u].z); x[u].w = __fadd_rn(x[u].w, y[u].w);
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      x[u].x = __fmul_rn(x[u].x, f); x[u].y = __fmul_rn(x[u].y, f);
      x[u].z = __fmul_rn(x[u].z, f); x[u].w = __fmul_rn(x[u].w, f);
      st_f4(a.dst + base + 1024 * u, x[u]);
    }
  }
  for (int64_t i = tiles * 4096 + 4 * (blockIdx.x * (int64_t)blockDim.x + threadIdx.x); i < a.n;
       i += 4 * (int64_t)gridDim.x * blockDim.x) {
    float4 x = ld_rw(a.dst + i);
    for (int s = 0; s < a.n_src; ++s) {
      const float4 y = ld_stream(a.src[s] + i);
      x.x = __fadd_rn(x.x, y.x); x.y = __fadd_rn(x.y, y.y); x.z = __fadd_rn(x.z, y.z); x.w = __fadd_rn(x.w, y.w);
    }
    x.x = __fmul_rn(x.x, f); x.y = __fmul_rn(x.y, f); x.z = __fmul_rn(x.z, f); x.w = __fmul_rn(x.w, f);
    st_f4(a.dst + i, x);
  }
}

__global__ void norm_finalize_kernel(const double* __restrict__ partials, int n, double max_norm,
                                     double* norm_out, float* coef_out) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  double s = 0.0;
  for (int i = 0; i < n; ++i) s += partials[i];  // index order: fixed
  const double norm = sqrt(s);
  *norm_out = norm;
  double c = 1.0;
  if (max_norm > 0.0) {
    c = max_norm / (norm + 1e-6);
    if (c > 1.0) c = 1.0;
  }
  *coef_out = (float)c;
}

__global__ void fold_partials_kernel(const double* __restrict__ all, int world, int n, int w_g,
                                     double* __restrict__ out) {
  for (int x = threadIdx.x; x < n; x += blockDim.x) {
    double s = all[x];
    if (x >= w_g && x < n - 1)
      for (int r = 1; r < world; ++r) s += all[(int64_t)r * n + x];  // rank order: fixed
    out[x] = s;
  }
}

int g_sm_count = 0;
__host__ std::atomic<int64_t>& launch_counter() {
  static std::atomic<int64_t> n{0};
  return n;
}

}  // namespace

int64_t launches() { return launch_counter().load(); }

int sm_count() {
  if (g_sm_count == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sm_count, cudaDevAttrMultiProcessorCount, dev);
    if (g_sm_count <= 0) g_sm_count = 148;
  }
  return g_sm_count;
}

namespace {
int env_int(const char* name, int dflt) {
  const char* e = getenv(name);
  return e ? atoi(e) : dflt;
}
}  // namespace

bool k2_dynamic() {
  static const bool dyn = [] {
    const char* e = getenv("SH_K2_SCHED");
    return !(e && strcmp(e, "static") == 0);
  }();
  return dyn;
}

cudaError_t adamw_multi(K2Args& a, cudaStream_t st, int* grid_out) {
  static const int U = env_int("SH_K2_U", 4) == 2 ? 2 : 4;  // U=4: 0.93 vs 0.89 of HBM peak (profiles/r01_kernels_microbench.txt)
  static const int bps = env_int("SH_K2_BPS", 4);
  // SH_K2_IMPL: "bulk4k" / "bulk2k" = bulk-copy pipeline (4096-element items, 1 block/SM, or
  // 2048-element items, 2 blocks/SM); "ldg3" = register-staged kernel capped at 80 registers (3
  // blocks/SM); "dyn2" = dynamic schedule at 2 blocks/SM; default: register-staged, dynamic schedule,
  // 3 blocks/SM when the caller passes counters (SH_K2_SCHED=static: never), else static, 2 blocks/SM
  static const int impl = [] {
    const char* e = getenv("SH_K2_IMPL");
    if (!e) return 0;
    if (strcmp(e, "bulk4k") == 0 || strcmp(e, "bulk") == 0) return 1;
    if (strcmp(e, "bulk2k") == 0) return 2;
    if (strcmp(e, "ldg3") == 0) return 3;
    if (strcmp(e, "dyn2") == 0) return 4;
    return 0;
  }();
  if (impl == 1 || impl == 2) {
    const int item = impl == 1 ? 4096 : 2048;
    a.item_start[0] = 0;
    for (int i = 0; i < a.n_entries; ++i) a.item_start[i + 1] = a.item_start[i] + (a.e[i].n + item - 1) / item;
    const int64_t items = a.item_start[a.n_entries];
    if (items == 0) return cudaSuccess;
    static bool attr_done = false;
    if (!attr_done) {
      cudaFuncSetAttribute(k2_adamw_bulk_kernel<true, 4096, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bulk_smem<4096>());
      cudaFuncSetAttribute(k2_adamw_bulk_kernel<false, 4096, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bulk_smem<4096>());
      cudaFuncSetAttribute(k2_adamw_bulk_kernel<true, 2048, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bulk_smem<2048>());
      cudaFuncSetAttribute(k2_adamw_bulk_kernel<false, 2048, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bulk_smem<2048>());
      attr_done = true;
    }
    const int64_t cap = (int64_t)sm_count() * (impl == 1 ? 1 : 2);
    const int grid = (int)(items < cap ? items : cap);
    if (grid_out) *grid_out = grid;
    launch_counter()++;
    if (impl == 1) {
      if (a.out_bf16) k2_adamw_bulk_kernel<true, 4096, 1><<<grid, kBulkThreads, bulk_smem<4096>(), st>>>(a);
      else k2_adamw_bulk_kernel<false, 4096, 1><<<grid, kBulkThreads, bulk_smem<4096>(), st>>>(a);
    } else {
      if (a.out_bf16) k2_adamw_bulk_kernel<true, 2048, 2><<<grid, kBulkThreads, bulk_smem<2048>(), st>>>(a);
      else k2_adamw_bulk_kernel<false, 2048, 2><<<grid, kBulkThreads, bulk_smem<2048>(), st>>>(a);
    }
    return cudaGetLastError();
  }
  const int64_t chunk = 1024 * U;
  a.item_start[0] = 0;
  for (int i = 0; i < a.n_entries; ++i) a.item_start[i + 1] = a.item_start[i] + (a.e[i].n + chunk - 1) / chunk;
  const int64_t items = a.item_start[a.n_entries];
  if (items == 0) return cudaSuccess;
  // Persistent-style grid: bps resident 256-thread blocks per SM, never more blocks than items.
  const int64_t cap = (int64_t)sm_count() * (bps > 0 ? bps : 4);
  const int grid = (int)(items < cap ? items : cap);
  if (grid_out) *grid_out = grid;
  launch_counter()++;
  // Default with counters (the engine's K2): dynamic schedule, 80-register build, 3 resident blocks per
  // SM, grid = exactly the resident blocks.  Isolated h=4096 layer (201 M elements): 6.75 TB/s vs 6.03
  // static (2 blocks/SM, two static waves); beside a D2H copy (the live step's usual neighbour) 6.47 vs
  // 5.82 TB/s (profiles/r02_k2_contention.jsonl).  SH_K2_IMPL=dyn2: dynamic, 2 blocks/SM.
  if (a.sched != nullptr && (impl == 0 || impl == 3 || impl == 4) && U == 4) {
    if (items >= (int64_t)1 << 32) return cudaErrorInvalidValue;  // 32-bit counter
    // exactly the resident blocks (the occupancy of the chosen build): a late block would only find
    // the counter exhausted
    static const int per_sm = [] {
      int nb = 0;
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, impl != 4 ? k2_adamw_kernel<true, 4, 3, true>
                                                                       : k2_adamw_kernel<true, 4, 0, true>, 256, 0) != cudaSuccess ||
          nb <= 0) {
        cudaGetLastError();
        nb = impl != 4 ? 3 : 2;
      }
      return nb;
    }();
    const int64_t dcap = (int64_t)sm_count() * per_sm;
    const int dgrid = (int)(items < dcap ? items : dcap);
    if (grid_out) *grid_out = dgrid;
    if (impl != 4) {
      if (a.out_bf16) k2_adamw_kernel<true, 4, 3, true><<<dgrid, 256, 0, st>>>(a);
      else k2_adamw_kernel<false, 4, 3, true><<<dgrid, 256, 0, st>>>(a);
    } else {
      if (a.out_bf16) k2_adamw_kernel<true, 4, 0, true><<<dgrid, 256, 0, st>>>(a);
      else k2_adamw_kernel<false, 4, 0, true><<<dgrid, 256, 0, st>>>(a);
    }
  } else if (impl == 3) {
    if (a.out_bf16) k2_adamw_kernel<true, 4, 3><<<grid, 256, 0, st>>>(a);
    else k2_adamw_kernel<false, 4, 3><<<grid, 256, 0, st>>>(a);
  } else if (U == 4) {
    if (a.out_bf16) k2_adamw_kernel<true, 4><<<grid, 256, 0, st>>>(a);
    else k2_adamw_kernel<false, 4><<<grid, 256, 0, st>>>(a);
  } else {
    if (a.out_bf16) k2_adamw_kernel<true, 2><<<grid, 256, 0, st>>>(a);
    else k2_adamw_kernel<false, 2><<<grid, 256, 0, st>>>(a);
  }
  return cudaGetLastError();
}

cudaError_t adamw_split(const K2SplitArgs& a, cudaStream_t st) {
  if (a.n <= 0) return cudaSuccess;
  if (!a.sched) return cudaErrorInvalidValue;
  const int64_t items = (a.n + 4095) / 4096;
  if (items >= (int64_t)1 << 32) return cudaErrorInvalidValue;
  static const int per_sm = [] {
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k2_split_kernel, 256, 0) != cudaSuccess || nb <= 0) {
      cudaGetLastError();
      nb = 3;
    }
    return nb;
  }();
  const int64_t cap = (int64_t)sm_count() * per_sm;
  launch_counter()++;
  k2_split_kernel<<<(int)(items < cap ? items : cap), 256, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t cast_bf16(const float* src, uint16_t* dst, int64_t n, cudaStream_t st) {
  const int64_t n8 = n / 8;
  if (n8 == 0) return cudaSuccess;
  const int64_t cap = (int64_t)sm_count() * 8;
  const int64_t need = (n8 + 255) / 256;
  launch_counter()++;
  k1_cast_kernel<<<(int)(need < cap ? need : cap), 256, 0, st>>>(src, dst, n8);
  return cudaGetLastError();
}

cudaError_t sumsq(const float* g, int64_t n, double* scratch, double* out, cudaStream_t st) {
  const int64_t n4 = n / 4;
  if (n4 == 0) return cudaMemsetAsync(out, 0, sizeof(double), st);
  int64_t nb = (n4 + 4095) / 4096;  // >= 16 float4 per thread before the tail
  if (nb > kSumsqMaxBlocks) nb = kSumsqMaxBlocks;
  launch_counter()++;
  unsigned int* ticket = reinterpret_cast<unsigned int*>(scratch + kSumsqMaxBlocks);
  k3_sumsq_kernel<<<(int)nb, 256, 0, st>>>(g, n4, scratch, ticket, out);
  return cudaGetLastError();
}

cudaError_t exec_reduce(const K4Args& a, cudaStream_t st) {
  if (a.n <= 0 || a.n_src < 0) return cudaSuccess;
  const int64_t cap = (int64_t)sm_count() * 8;  // persistent: 8 x 256 threads per SM (44 regs)
  const int64_t need = (a.n + 4095) / 4096;
  launch_counter()++;
  k4_exec_reduce_kernel<<<(int)(need < cap ? need : cap), 256, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t norm_finalize(const double* partials, int n, double max_norm, double* norm_out,
                          float* coef_out, cudaStream_t st) {
  launch_counter()++;
  norm_finalize_kernel<<<1, 32, 0, st>>>(partials, n, max_norm, norm_out, coef_out);
  return cudaGetLastError();
}

}  // namespace kern
}  // namespace sh

namespace sh {
namespace kern {
cudaError_t fold_partials(const double* all, int world, int n, int w_g, double* out, cudaStream_t st) {
  launch_counter()++;
  fold_partials_kernel<<<1, 256, 0, st>>>(all, world, n, w_g, out);
  return cudaGetLastError();
}
}  // namespace kern
}  // namespace sh
