// GPT-2 block compute that drives the offload engine -- OUTSIDE THE HOT PATH (see sh_gpt.h).
//
// GEMMs: cuBLAS (bf16 or fp32 operands, fp32 accumulation, CUBLAS_COMPUTE_32F, fixed workspace,
// atomics disallowed => run-to-run bitwise reproducible; on sm_100 the bf16 GEMMs run on the
// tcgen05 tensor cores inside cuBLAS).  Attention runs as pointer-array batched GEMMs directly
// on the [N, 3h] qkv layout (no permute kernels); biases are folded into the GEMMs by a
// broadcast prefill + beta = 1 (one rounding of acc + bias).  The remaining SIMT kernels are
// HBM-bound and move 16-byte vectors (8 bf16 / 2 x 4 fp32) with fixed reduction orders.
// The math is DESIGN.md reading R1 / oracle/gpt_oracle.py (shared by definition, not code).
#include <cublasLt.h>
#include <cublas_v2.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>

#include <algorithm>
#include <atomic>
#include <type_traits>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>

#include "sh_gpt.h"

namespace {

thread_local std::string g_err;
std::atomic<int64_t> g_launches{0};
void seterr(const char* fmt, ...) {
  char b[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(b, sizeof(b), fmt, ap);
  va_end(ap);
  g_err = b;
}

using bf16 = __nv_bfloat16;
constexpr float kLnEps = 1e-5f;

__device__ __forceinline__ float tof(float x) { return x; }
__device__ __forceinline__ float tof(bf16 x) { return __bfloat162float(x); }
template <class T> __device__ __forceinline__ T fromf(float x);
template <> __device__ __forceinline__ float fromf<float>(float x) { return x; }
template <> __device__ __forceinline__ bf16 fromf<bf16>(float x) { return __float2bfloat16_rn(x); }

// 8-element vector load/store as floats (16 B for bf16, 2 x 16 B for fp32)
__device__ __forceinline__ void ld8(const float* p, float (&v)[8]) {
  const float4 a = reinterpret_cast<const float4*>(p)[0], b = reinterpret_cast<const float4*>(p)[1];
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}
__device__ __forceinline__ void ld8(const bf16* p, float (&v)[8]) {
  const uint4 u = *reinterpret_cast<const uint4*>(p);
  const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    v[2 * i] = __uint_as_float(w[i] << 16);
    v[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
  }
}
__device__ __forceinline__ void st8(float* p, const float (&v)[8]) {
  reinterpret_cast<float4*>(p)[0] = make_float4(v[0], v[1], v[2], v[3]);
  reinterpret_cast<float4*>(p)[1] = make_float4(v[4], v[5], v[6], v[7]);
}
__device__ __forceinline__ void st8(bf16* p, const float (&v)[8]) {
  uint32_t w[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t lo = __bfloat16_as_ushort(__float2bfloat16_rn(v[2 * i]));
    const uint32_t hi = __bfloat16_as_ushort(__float2bfloat16_rn(v[2 * i + 1]));
    w[i] = lo | (hi << 16);
  }
  *reinterpret_cast<uint4*>(p) = make_uint4(w[0], w[1], w[2], w[3]);
}

__device__ __forceinline__ float warp_sum(float x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}
__device__ __forceinline__ float warp_max(float x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x = fmaxf(x, __shfl_xor_sync(0xffffffffu, x, o));
  return x;
}
template <int NT>
__device__ __forceinline__ float block_reduce(float x, bool is_max) {
  __shared__ float sh[NT / 32];
  x = is_max ? warp_max(x) : warp_sum(x);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();
  if (l == 0) sh[w] = x;
  __syncthreads();
  float r = l < NT / 32 ? sh[l] : (is_max ? -INFINITY : 0.f);
  r = is_max ? warp_max(r) : warp_sum(r);
  return r;  // every warp computes the same fixed-order result
}

#define GRID_STRIDE(i, n) for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n); i += (int64_t)gridDim.x * blockDim.x)

// ------------------------------------------------------------------------------ kernels
template <class T>
__global__ void embed_fwd(const int* tok, const T* wte, const T* wpe, float* x, int S, int h) {
  const int n = blockIdx.x;  // token row b*S+s
  const int b = n / S, s = n % S;
  const int t = tok[b * (S + 1) + s];
  for (int c = 8 * threadIdx.x; c < h; c += 8 * blockDim.x) {
    float a[8], p[8];
    ld8(wte + (int64_t)t * h + c, a);
    ld8(wpe + (int64_t)s * h + c, p);
#pragma unroll
    for (int i = 0; i < 8; ++i) a[i] += p[i];
    st8(x + (int64_t)n * h + c, a);
  }
}

// one warp per row; two-pass statistics (mean, then centred variance) in fp32
template <class T>
__global__ void ln_fwd(const float* x, const T* g, const T* b, T* out, float* mean, float* rstd, int N, int h) {
  const int row = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= N) return;
  const float* xr = x + (int64_t)row * h;
  float s = 0.f;
  // unrolled for memory-level parallelism; each lane still accumulates in index order
#pragma unroll 4
  for (int c = 8 * lane; c < h; c += 256) {
    float v[8];
    ld8(xr + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) s += v[i];
  }
  const float mu = warp_sum(s) / h;
  float var = 0.f;
  // unrolled for memory-level parallelism; each lane still accumulates in index order
#pragma unroll 4
  for (int c = 8 * lane; c < h; c += 256) {
    float v[8];
    ld8(xr + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) var += (v[i] - mu) * (v[i] - mu);
  }
  const float rs = 1.0f / sqrtf(warp_sum(var) / h + kLnEps);
  T* o = out + (int64_t)row * h;
  // unrolled for memory-level parallelism; each lane still accumulates in index order
#pragma unroll 4
  for (int c = 8 * lane; c < h; c += 256) {
    float v[8], gg[8], bb[8];
    ld8(xr + c, v);
    ld8(g + c, gg);
    ld8(b + c, bb);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = (v[i] - mu) * rs * gg[i] + bb[i];
    st8(o + c, v);
  }
  if (lane == 0) {
    mean[row] = mu;
    rstd[row] = rs;
  }
}

// Register-cached LN (h <= 8192): one 128-thread block per row, thread t holds elements
// 8t + 1024k (k < K) of the row, so x (and dy) are read from DRAM once; the two-pass warp-per-row
// kernels re-read the row from DRAM (measured: 2x the algorithmic bytes at h 4096).  Block sums
// are a fixed tree (warp shuffle, then the 4 warp partials in order): deterministic.
__device__ __forceinline__ float block_sum128(float x, float* red) {
  x = warp_sum(x);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = x;
  __syncthreads();
  const float r = (red[0] + red[1]) + (red[2] + red[3]);
  __syncthreads();  // red is reused by the next reduction
  return r;
}

template <class T, int K>
__global__ void __launch_bounds__(128) ln_fwd_reg(const float* x, const T* g, const T* b, T* out, float* mean,
                                                  float* rstd, int N, int h) {
  __shared__ float red[4];
  const int row = blockIdx.x;
  const float* xr = x + (int64_t)row * h;
  float v[K][8];
  float s = 0.f;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const int c = 8 * threadIdx.x + 1024 * k;
    if (c < h) {
      ld8(xr + c, v[k]);
#pragma unroll
      for (int i = 0; i < 8; ++i) s += v[k][i];
    }
  }
  const float mu = block_sum128(s, red) / h;
  float var = 0.f;
#pragma unroll
  for (int k = 0; k < K; ++k)
    if (8 * threadIdx.x + 1024 * k < h)
#pragma unroll
      for (int i = 0; i < 8; ++i) var += (v[k][i] - mu) * (v[k][i] - mu);
  const float rs = 1.0f / sqrtf(block_sum128(var, red) / h + kLnEps);
  T* o = out + (int64_t)row * h;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const int c = 8 * threadIdx.x + 1024 * k;
    if (c < h) {
      float gg[8], bb[8];
      ld8(g + c, gg);
      ld8(b + c, bb);
#pragma unroll
      for (int i = 0; i < 8; ++i) v[k][i] = (v[k][i] - mu) * rs * gg[i] + bb[i];
      st8(o + c, v[k]);
    }
  }
  if (threadIdx.x == 0) {
    mean[row] = mu;
    rstd[row] = rs;
  }
}

template <class T, int K>
__global__ void __launch_bounds__(128) ln_bwd_reg(const float* dy, const float* x, const float* mean,
                                                  const float* rstd, const T* g, float* dres, float* tmp, int N,
                                                  int h) {
  __shared__ float red[4];
  const int row = blockIdx.x;
  const float* dr = dy + (int64_t)row * h;
  const float* xr = x + (int64_t)row * h;
  const float mu = mean[row], rs = rstd[row];
  float d[K][8], xh[K][8];
  float a = 0.f, bb = 0.f;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const int c = 8 * threadIdx.x + 1024 * k;
    if (c < h) {
      float gg[8];
      ld8(dr + c, d[k]);
      ld8(xr + c, xh[k]);
      ld8(g + c, gg);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        xh[k][i] = (xh[k][i] - mu) * rs;
        const float dxh = d[k][i] * gg[i];
        a += dxh;
        bb += dxh * xh[k][i];
      }
    }
  }
  a = block_sum128(a, red) / h;
  bb = block_sum128(bb, red) / h;
  float* o = dres + (int64_t)row * h;
  float* t = tmp + (int64_t)row * h;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const int c = 8 * threadIdx.x + 1024 * k;
    if (c < h) {
      float gg[8], ov[8], tv[8];
      ld8(g + c, gg);
      ld8(o + c, ov);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        ov[i] += rs * (d[k][i] * gg[i] - a - xh[k][i] * bb);
        tv[i] = d[k][i] * xh[k][i];
      }
      st8(o + c, ov);
      st8(t + c, tv);
    }
  }
}

// dres += LN backward(dy); tmp = dy * xhat (for dgamma); dbeta = colsum(dy) done by cuBLAS
template <class T>
__global__ void ln_bwd(const float* dy, const float* x, const float* mean, const float* rstd, const T* g,
                       float* dres, float* tmp, int N, int h) {
  const int row = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= N) return;
  const float* dr = dy + (int64_t)row * h;
  const float* xr = x + (int64_t)row * h;
  const float mu = mean[row], rs = rstd[row];
  float a = 0.f, bb = 0.f;
  // unrolled for memory-level parallelism; each lane still accumulates in index order
#pragma unroll 4
  for (int c = 8 * lane; c < h; c += 256) {
    float d[8], xv[8], gg[8];
    ld8(dr + c, d);
    ld8(xr + c, xv);
    ld8(g + c, gg);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const float dxh = d[i] * gg[i];
      a += dxh;
      bb += dxh * ((xv[i] - mu) * rs);
    }
  }
  a = warp_sum(a) / h;
  bb = warp_sum(bb) / h;
  float* o = dres + (int64_t)row * h;
  float* t = tmp + (int64_t)row * h;
  // unrolled for memory-level parallelism; each lane still accumulates in index order
#pragma unroll 4
  for (int c = 8 * lane; c < h; c += 256) {
    float d[8], xv[8], gg[8], ov[8], tv[8];
    ld8(dr + c, d);
    ld8(xr + c, xv);
    ld8(g + c, gg);
    ld8(o + c, ov);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const float xh = (xv[i] - mu) * rs;
      ov[i] += rs * (d[i] * gg[i] - a - xh * bb);
      tv[i] = d[i] * xh;
    }
    st8(o + c, ov);
    st8(t + c, tv);
  }
}

// out[r, :] = bias (T) or x[r, :] + bias (fp32 residual); C % 8 == 0
template <class T>
__global__ void bias_fill(T* out, const T* bias, int C, int64_t n8) {
  const int c8 = C / 8;
  GRID_STRIDE(j, n8) {
    float v[8];
    ld8(bias + (j % c8) * 8, v);
    st8(out + 8 * j, v);
  }
}
template <class T>
__global__ void resid_bias(const float* x, const T* bias, float* out, int C, int64_t n8) {
  const int c8 = C / 8;
  GRID_STRIDE(j, n8) {
    float v[8], b[8];
    ld8(x + 8 * j, v);
    ld8(bias + (j % c8) * 8, b);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] += b[i];
    st8(out + 8 * j, v);
  }
}

// tanh: the accurate tanhf in fp32 mode; MUFU.TANH (tanh.approx.f32, |rel err| ~ 2^-11) for bf16
// activations, whose own rounding is 2^-9 -- the accurate tanhf made the GELU kernels
// issue-bound (4 TB/s at h 4096)
template <class T>
__device__ __forceinline__ float tanh_t(float x) {
  if constexpr (std::is_same<T, bf16>::value) {
    float y;
    asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
  } else {
    return tanhf(x);
  }
}
template <class T>
__device__ __forceinline__ float gelu_f(float u) {
  const float k = 0.7978845608028654f;  // sqrt(2/pi)
  return 0.5f * u * (1.0f + tanh_t<T>(k * (u + 0.044715f * u * u * u)));
}
template <class T>
__device__ __forceinline__ float gelu_grad(float u) {
  const float k = 0.7978845608028654f;
  const float t = tanh_t<T>(k * (u + 0.044715f * u * u * u));
  return 0.5f * (1.0f + t) + 0.5f * u * (1.0f - t * t) * k * (1.0f + 3.0f * 0.044715f * u * u);
}

template <class T>
__global__ void gelu_fwd(const T* pre, T* act, int64_t n8) {
  GRID_STRIDE(j, n8) {
    float v[8];
    ld8(pre + 8 * j, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = gelu_f<T>(v[i]);
    st8(act + 8 * j, v);
  }
}
template <class T>
__global__ void gelu_bwd(T* d, const T* pre, int64_t n8) {
  GRID_STRIDE(j, n8) {
    float v[8], u[8];
    ld8(d + 8 * j, v);
    ld8(pre + 8 * j, u);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] *= gelu_grad<T>(u[i]);
    st8(d + 8 * j, v);
  }
}
template <class T>
__global__ void cast_f2t(const float* a, T* o, int64_t n8) {
  GRID_STRIDE(j, n8) {
    float v[8];
    ld8(a + 8 * j, v);
    st8(o + 8 * j, v);
  }
}
template <class T>
__global__ void fill_ones(T* o, int64_t n) {
  GRID_STRIDE(i, n) o[i] = fromf<T>(1.0f);
}

// Causal softmax, one warp per score row; lane owns 8-column chunks lane, lane+32, ...
// (NCH = chunks per lane).  Chunks entirely above the diagonal are never read (exact zeros).
template <class T, int NCH>
__global__ void softmax_causal(const float* sc, T* p, int S, int64_t rows) {
  const int64_t row = blockIdx.x * (int64_t)(blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= rows) return;
  const int r = (int)(row % S);
  const float* s = sc + row * S;
  T* o = p + row * S;
  float v[NCH][8];
  float m = -INFINITY;
#pragma unroll
  for (int k = 0; k < NCH; ++k) {
    const int c0 = 8 * (lane + 32 * k);
    if (c0 < S && c0 <= r) {
      ld8(s + c0, v[k]);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        if (c0 + i > r) v[k][i] = -INFINITY;
        m = fmaxf(m, v[k][i]);
      }
    }
  }
  m = warp_max(m);
  float z = 0.f;
#pragma unroll
  for (int k = 0; k < NCH; ++k) {
    const int c0 = 8 * (lane + 32 * k);
    if (c0 < S && c0 <= r) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        v[k][i] = c0 + i <= r ? expf(v[k][i] - m) : 0.f;
        z += v[k][i];
      }
    }
  }
  const float inv = 1.0f / warp_sum(z);
#pragma unroll
  for (int k = 0; k < NCH; ++k) {
    const int c0 = 8 * (lane + 32 * k);
    if (c0 < S) {
      float w[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) w[i] = c0 <= r ? v[k][i] * inv : 0.f;
      st8(o + c0, w);
    }
  }
}

// dS = P * (dP - Σ dP*P), written in place over P (chunks above the diagonal stay 0)
template <class T, int NCH>
__global__ void softmax_bwd(T* p, const float* dp, int S, int64_t rows) {
  const int64_t row = blockIdx.x * (int64_t)(blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= rows) return;
  const int r = (int)(row % S);
  T* pr = p + row * S;
  const float* d = dp + row * S;
  float pv[NCH][8], dv[NCH][8];
  float a = 0.f;
#pragma unroll
  for (int k = 0; k < NCH; ++k) {
    const int c0 = 8 * (lane + 32 * k);
    if (c0 < S && c0 <= r) {
      ld8(pr + c0, pv[k]);
      ld8(d + c0, dv[k]);
#pragma unroll
      for (int i = 0; i < 8; ++i) a += pv[k][i] * dv[k][i];  // P == 0 above the diagonal
    }
  }
  a = warp_sum(a);
#pragma unroll
  for (int k = 0; k < NCH; ++k) {
    const int c0 = 8 * (lane + 32 * k);
    if (c0 < S && c0 <= r) {
#pragma unroll
      for (int i = 0; i < 8; ++i) pv[k][i] = pv[k][i] * (dv[k][i] - a);
      st8(pr + c0, pv[k]);
    }
  }
}

// cross entropy per row (block of 512): loss_n, dlogits_n = (softmax - onehot)/Ntot
template <class T>
__global__ void __launch_bounds__(512) ce_fwd_bwd(const float* logits, const int* tok, int S, int V, float inv_n,
                                                  float* row_loss, T* dlogits) {
  const int64_t n = blockIdx.x;
  const int b = (int)(n / S), s = (int)(n % S);
  const int tgt = tok[b * (S + 1) + s + 1];
  const float* l = logits + n * V;
  float m = -INFINITY;
  for (int c = 8 * threadIdx.x; c < V; c += 8 * 512) {
    float v[8];
    ld8(l + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) m = fmaxf(m, v[i]);
  }
  m = block_reduce<512>(m, true);
  float z = 0.f;
  for (int c = 8 * threadIdx.x; c < V; c += 8 * 512) {
    float v[8];
    ld8(l + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) z += expf(v[i] - m);
  }
  z = block_reduce<512>(z, false);
  const float inv = 1.0f / z;
  const float lt = l[tgt];
  __syncthreads();  // all reads of l[] done before an in-place (fp32) overwrite
  T* d = dlogits + n * V;
  for (int c = 8 * threadIdx.x; c < V; c += 8 * 512) {
    float v[8];
    ld8(l + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      float pr = expf(v[i] - m) * inv;
      if (c + i == tgt) pr -= 1.0f;
      v[i] = pr * inv_n;
    }
    st8(d + c, v);
  }
  if (threadIdx.x == 0) row_loss[n] = logf(z) + m - lt;
}

__global__ void mean_fixed(const float* a, int n, float scale, float* out) {
  float s = 0.f;
  for (int i = threadIdx.x; i < n; i += 512) s += a[i];
  s = block_reduce<512>(s, false);
  if (threadIdx.x == 0) *out = s * scale;
}

__global__ void gather_tokens(const int* tok, int S, int N, int* keys, int* vals) {
  const int n = blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= N) return;
  keys[n] = tok[(n / S) * (S + 1) + n % S];
  vals[n] = n;
}

// dwte[v] += Σ rows of dx at positions with token v, in increasing position order
__global__ void embed_bwd_wte(const int* keys, const int* vals, const float* dx, float* dwte, int N, int h) {
  const int i = blockIdx.x;
  const int v = keys[i];
  if (i > 0 && keys[i - 1] == v) return;  // not the start of a segment
  for (int c = threadIdx.x; c < h; c += blockDim.x) {
    float acc = dwte[(int64_t)v * h + c];
    for (int j = i; j < N && keys[j] == v; ++j) acc += dx[(int64_t)vals[j] * h + c];
    dwte[(int64_t)v * h + c] = acc;
  }
}
__global__ void embed_bwd_wpe(const float* dx, float* dwpe, int B, int S, int h) {
  const int s = blockIdx.x;
  for (int c = threadIdx.x; c < h; c += blockDim.x) {
    float acc = dwpe[(int64_t)s * h + c];
    for (int b = 0; b < B; ++b) acc += dx[((int64_t)b * S + s) * h + c];
    dwpe[(int64_t)s * h + c] = acc;
  }
}

// pointer arrays of the per-(batch, head) attention operands on the [N, 3h] / [N, h] layouts
__global__ void build_attn_ptrs(void** P, char* qkv, char* scores, char* probs, char* att, char* datt,
                                char* dqkv, int B, int nh, int S, int h, int es) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int BH = B * nh;
  if (i >= BH) return;
  const int b = i / nh, hd_i = i % nh, hd = h / nh;
  const int64_t row3 = (int64_t)b * S * 3 * h, row1 = (int64_t)b * S * h, col = (int64_t)hd_i * hd;
  P[0 * BH + i] = qkv + es * (row3 + col);
  P[1 * BH + i] = qkv + es * (row3 + h + col);
  P[2 * BH + i] = qkv + es * (row3 + 2 * h + col);
  P[3 * BH + i] = scores + 4 * (int64_t)i * S * S;
  P[4 * BH + i] = probs + es * (int64_t)i * S * S;
  P[5 * BH + i] = att + es * (row1 + col);
  P[6 * BH + i] = datt + es * (row1 + col);
  P[7 * BH + i] = dqkv + es * (row3 + col);
  P[8 * BH + i] = dqkv + es * (row3 + h + col);
  P[9 * BH + i] = dqkv + es * (row3 + 2 * h + col);
}

int grid_for(int64_t total, int threads = 256) {
  int64_t g = (total + threads - 1) / threads;
  const int64_t cap = 148 * 16;
  return (int)(g < cap ? (g > 0 ? g : 1) : cap);
}

// LN launchers: the register-cached kernels for h <= 8192 (K = ceil(h / 1024) groups of 8 per thread)
template <class T>
void launch_ln_fwd(cudaStream_t st, const float* x, const T* g, const T* b, T* out, float* m, float* r, int N, int h) {
  static const bool reg = !(getenv("SH_GPT_LN_REG") && getenv("SH_GPT_LN_REG")[0] == '0');  // A/B switch
  const int K = reg ? (h + 1023) / 1024 : 0;
  g_launches++;
  switch (K) {
#define LNF(k) case k: ln_fwd_reg<T, k><<<N, 128, 0, st>>>(x, g, b, out, m, r, N, h); break;
    LNF(1) LNF(2) LNF(3) LNF(4) LNF(5) LNF(6) LNF(7) LNF(8)
#undef LNF
    default: ln_fwd<T><<<(N + 7) / 8, 256, 0, st>>>(x, g, b, out, m, r, N, h);
  }
}
template <class T>
void launch_ln_bwd(cudaStream_t st, const float* dy, const float* x, const float* m, const float* r, const T* g,
                   float* dres, float* tmp, int N, int h) {
  static const bool reg = !(getenv("SH_GPT_LN_REG") && getenv("SH_GPT_LN_REG")[0] == '0');  // A/B switch
  const int K = reg ? (h + 1023) / 1024 : 0;
  g_launches++;
  switch (K) {
#define LNB(k) case k: ln_bwd_reg<T, k><<<N, 128, 0, st>>>(dy, x, m, r, g, dres, tmp, N, h); break;
    LNB(1) LNB(2) LNB(3) LNB(4) LNB(5) LNB(6) LNB(7) LNB(8)
#undef LNB
    default: ln_bwd<T><<<(N + 7) / 8, 256, 0, st>>>(dy, x, m, r, g, dres, tmp, N, h);
  }
}

}  // namespace

struct gpt_ctx {
  gpt_config cfg{};
  bool bf16 = true;
  int es = 2;  // element size of T
  cudaDataType_t dt = CUDA_R_16BF;
  cudaStream_t st = nullptr;
  cublasHandle_t cb = nullptr;
  void* ws = nullptr;
  size_t ws_bytes = 64u << 20;
  int B = 0, N = 0, S = 0, h = 0, nh = 0, V = 0, L = 0;
  int ptrB = -1;
  int64_t maxN = 0;
  std::vector<void*> allocs;
  int64_t bytes = 0;
  float* x = nullptr;  // (L+1) checkpoints
  void *ln1, *ln2, *lnf, *qkv, *probs, *att, *fc_pre, *fc_act, *dy, *d4h, *datt, *dqkv, *ones_t, *dlogits;
  float *ln1_m, *ln1_r, *ln2_m, *ln2_r, *lnf_m, *lnf_r, *scores, *x_mid, *dres, *dln, *tmp, *logits, *row_loss, *ones_f;
  void** aptr = nullptr;  // 10 x BH attention operand pointers
  int *keys, *vals, *keys2, *vals2;
  void* cub_tmp = nullptr;
  size_t cub_bytes = 0;
  // bf16 path: cuBLASLt GEMMs with fused epilogues (bias; bias + GELU with the pre-activation kept
  // for the backward; GELU gradient) replace the bias-fill / GELU SIMT passes
  cublasLtHandle_t lt = nullptr;
  int use_lt = 0;  // bit 1: qkv bias epilogue, 2: fc bias + GELU, 4: dGELU (SH_GPT_LT, default all)
  struct LtAlgo {
    int64_t key[7];
    cublasLtMatmulAlgo_t algo;
  };
  std::vector<LtAlgo> lt_algos;
};

namespace {

int alloc(gpt_ctx* c, void** p, int64_t bytes) {
  bytes = (bytes + 255) / 256 * 256;
  if (cudaMalloc(p, bytes) != cudaSuccess) {
    cudaGetLastError();
    seterr("gpt: cudaMalloc(%lld) failed", (long long)bytes);
    return -3;
  }
  c->allocs.push_back(*p);
  c->bytes += bytes;
  return 0;
}

#define CK(x)                                                     \
  do {                                                            \
    cudaError_t e_ = (x);                                         \
    if (e_ != cudaSuccess) {                                      \
      seterr("gpt: %s: %s", #x, cudaGetErrorString(e_));          \
      return -2;                                                  \
    }                                                             \
  } while (0)
#define CB(x)                                                     \
  do {                                                            \
    cublasStatus_t s_ = (x);                                      \
    if (s_ != CUBLAS_STATUS_SUCCESS) {                            \
      seterr("gpt: %s: cublas status %d", #x, (int)s_);           \
      return -4;                                                  \
    }                                                             \
  } while (0)

// Row-major C[M,N] (row stride ldc) = alpha op(A) op(B) + beta C.  A is [M,K] (or stored [K,M]
// if tA) with row stride lda; B is [K,N] (or stored [N,K] if tB) with row stride ldb.
// Column-major cuBLAS computes C^T = op(B)^T op(A)^T.
cublasStatus_t gemm(gpt_ctx* c, bool tA, bool tB, int M, int N, int K, float alpha, const void* A, cudaDataType_t ta,
                    int lda, const void* B, cudaDataType_t tb, int ldb, float beta, void* C, cudaDataType_t tc, int ldc) {
  return cublasGemmEx(c->cb, tB ? CUBLAS_OP_T : CUBLAS_OP_N, tA ? CUBLAS_OP_T : CUBLAS_OP_N, N, M, K, &alpha, B, tb,
                      ldb, A, ta, lda, &beta, C, tc, ldc, CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
}
cublasStatus_t rm_gemm(gpt_ctx* c, bool tA, bool tB, int M, int N, int K, float alpha, const void* A,
                       cudaDataType_t ta, const void* B, cudaDataType_t tb, float beta, void* C, cudaDataType_t tc) {
  return gemm(c, tA, tB, M, N, K, alpha, A, ta, tA ? M : K, B, tb, tB ? K : N, beta, C, tc, N);
}
// Row-major bf16 D[M x N] = op(A)[M x K] op(B)[K x N] through cuBLASLt with an epilogue:
//   CUBLASLT_EPILOGUE_BIAS           D = AB + bias[N]
//   CUBLASLT_EPILOGUE_GELU_AUX_BIAS  aux = AB + bias[N] (pre-activation, kept for the backward),
//                                    D = GELU(aux)
//   CUBLASLT_EPILOGUE_DGELU          D = AB * GELU'(aux)
// Same column-major mapping as gemm(): D^T = op(B)^T op(A)^T.  fp32 accumulate; the algorithm is
// chosen once per shape by the heuristic and cached (same shape -> same algorithm -> same bits).
cublasStatus_t lt_gemm(gpt_ctx* c, bool tA, bool tB, int M, int N, int K, const void* A, const void* B, void* D,
                       cublasLtEpilogue_t epi, const void* bias, void* aux) {
  const cublasOperation_t ta = tB ? CUBLAS_OP_T : CUBLAS_OP_N, tb = tA ? CUBLAS_OP_T : CUBLAS_OP_N;
  cublasLtMatmulDesc_t op = nullptr;
  cublasLtMatrixLayout_t la = nullptr, lb = nullptr, ld = nullptr;
  cublasStatus_t st = cublasLtMatmulDescCreate(&op, CUBLAS_COMPUTE_32F, CUDA_R_32F);
  auto set = [&](cublasLtMatmulDescAttributes_t a, const void* v, size_t n) {
    if (st == CUBLAS_STATUS_SUCCESS) st = cublasLtMatmulDescSetAttribute(op, a, v, n);
  };
  set(CUBLASLT_MATMUL_DESC_TRANSA, &ta, sizeof(ta));
  set(CUBLASLT_MATMUL_DESC_TRANSB, &tb, sizeof(tb));
  set(CUBLASLT_MATMUL_DESC_EPILOGUE, &epi, sizeof(epi));
  if (bias) set(CUBLASLT_MATMUL_DESC_BIAS_POINTER, &bias, sizeof(bias));
  if (aux) {
    const int64_t ald = N;
    const int32_t adt = CUDA_R_16BF;
    set(CUBLASLT_MATMUL_DESC_EPILOGUE_AUX_POINTER, &aux, sizeof(aux));
    set(CUBLASLT_MATMUL_DESC_EPILOGUE_AUX_LD, &ald, sizeof(ald));
    set(CUBLASLT_MATMUL_DESC_EPILOGUE_AUX_DATA_TYPE, &adt, sizeof(adt));
  }
  if (st == CUBLAS_STATUS_SUCCESS)
    st = cublasLtMatrixLayoutCreate(&la, CUDA_R_16BF, ta == CUBLAS_OP_T ? K : N, ta == CUBLAS_OP_T ? N : K, tB ? K : N);
  if (st == CUBLAS_STATUS_SUCCESS)
    st = cublasLtMatrixLayoutCreate(&lb, CUDA_R_16BF, tb == CUBLAS_OP_T ? M : K, tb == CUBLAS_OP_T ? K : M, tA ? M : K);
  if (st == CUBLAS_STATUS_SUCCESS) st = cublasLtMatrixLayoutCreate(&ld, CUDA_R_16BF, N, M, N);
  const int64_t key[7] = {M, N, K, tA, tB, (int64_t)epi, (int64_t)(bias != nullptr)};
  const cublasLtMatmulAlgo_t* algo = nullptr;
  for (auto& a : c->lt_algos)
    if (std::equal(key, key + 7, a.key)) algo = &a.algo;
  if (st == CUBLAS_STATUS_SUCCESS && !algo) {
    cublasLtMatmulPreference_t pref = nullptr;
    st = cublasLtMatmulPreferenceCreate(&pref);
    const uint64_t wsb = c->ws_bytes;
    if (st == CUBLAS_STATUS_SUCCESS)
      st = cublasLtMatmulPreferenceSetAttribute(pref, CUBLASLT_MATMUL_PREF_MAX_WORKSPACE_BYTES, &wsb, sizeof(wsb));
    cublasLtMatmulHeuristicResult_t res{};
    int n_res = 0;
    if (st == CUBLAS_STATUS_SUCCESS)
      st = cublasLtMatmulAlgoGetHeuristic(c->lt, op, la, lb, ld, ld, pref, 1, &res, &n_res);
    if (pref) cublasLtMatmulPreferenceDestroy(pref);
    if (st == CUBLAS_STATUS_SUCCESS && n_res < 1) st = CUBLAS_STATUS_NOT_SUPPORTED;
    if (st == CUBLAS_STATUS_SUCCESS) {
      gpt_ctx::LtAlgo e;
      std::copy(key, key + 7, e.key);
      e.algo = res.algo;
      c->lt_algos.push_back(e);
      algo = &c->lt_algos.back().algo;
    }
  }
  const float one = 1.f, zero = 0.f;
  if (st == CUBLAS_STATUS_SUCCESS)
    st = cublasLtMatmul(c->lt, op, &one, B, la, A, lb, &zero, D, ld, D, ld, algo, c->ws, c->ws_bytes, c->st);
  if (ld) cublasLtMatrixLayoutDestroy(ld);
  if (lb) cublasLtMatrixLayoutDestroy(lb);
  if (la) cublasLtMatrixLayoutDestroy(la);
  if (op) cublasLtMatmulDescDestroy(op);
  return st;
}

// batched over pointer arrays (attention): operand pointer arrays Ap, Bp, Cp on the device
cublasStatus_t gemm_ptr(gpt_ctx* c, bool tA, bool tB, int M, int N, int K, float alpha, void* const* Ap,
                        cudaDataType_t ta, int lda, void* const* Bp, cudaDataType_t tb, int ldb, float beta,
                        void* const* Cp, cudaDataType_t tc, int ldc, int batch) {
  return cublasGemmBatchedEx(c->cb, tB ? CUBLAS_OP_T : CUBLAS_OP_N, tA ? CUBLAS_OP_T : CUBLAS_OP_N, N, M, K, &alpha,
                             (const void* const*)Bp, tb, ldb, (const void* const*)Ap, ta, lda, &beta, Cp, tc, ldc,
                             batch, CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
}

// out[C] (fp32) = Σ_rows X[rows, C] (fixed-order cuBLAS reduction)
int colsum(gpt_ctx* c, const void* X, bool x_is_f32, int rows, int C, float* out) {
  if (x_is_f32 || !c->bf16) {
    const float one = 1.f, zero = 0.f;
    CB(cublasSgemv(c->cb, CUBLAS_OP_N, C, rows, &one, (const float*)X, C, c->ones_f, 1, &zero, out, 1));
  } else {
    CB(rm_gemm(c, false, false, 1, C, rows, 1.f, c->ones_t, c->dt, X, c->dt, 0.f, out, CUDA_R_32F));
  }
  return 0;
}

template <class T, int NCH>
void launch_softmax(gpt_ctx* c, int64_t rows, bool bwd) {
  if (bwd)
    (g_launches++, 0), softmax_bwd<T, NCH><<<(int)((rows + 7) / 8), 256, 0, c->st>>>((T*)c->probs, c->scores, c->S, rows);
  else
    (g_launches++, 0), softmax_causal<T, NCH><<<(int)((rows + 7) / 8), 256, 0, c->st>>>(c->scores, (T*)c->probs, c->S, rows);
}
template <class T>
int softmax(gpt_ctx* c, int64_t rows, bool bwd) {
  const int nch = (c->S / 8 + 31) / 32;
  switch (nch) {
    case 1: launch_softmax<T, 1>(c, rows, bwd); break;
    case 2: launch_softmax<T, 2>(c, rows, bwd); break;
    case 4: launch_softmax<T, 4>(c, rows, bwd); break;
    case 8: launch_softmax<T, 8>(c, rows, bwd); break;
    default: seterr("gpt: seq %d unsupported (S/256 must be 1, 2, 4 or 8 chunks per lane)", c->S); return -1;
  }
  return 0;
}

void** AP(gpt_ctx* c, int k) { return c->aptr + (int64_t)k * c->B * c->nh; }
enum { PQ = 0, PK, PV, PS, PP, PO, PDO, PDQ, PDK, PDV };

// Block forward in three stages so a caller can substitute the attention core (stage 2):
//   fwd_qkv:  ln1, qkv = ln1 W_qkv^T + b_qkv                     -> c->qkv  [N, 3h]
//   fwd_attn: att = causal softmax(q k^T / sqrt(hd)) v (cuBLAS)   -> c->att  [N, h]
//   fwd_out:  x_mid = x + att W_o^T + b_o; ln2; MLP; x_out
template <class T>
int fwd_qkv(gpt_ctx* c, int l, void* const* P) {
  const int N = c->N, h = c->h;
  const cudaDataType_t dt = c->dt;
  const float* xin = c->x + (int64_t)l * c->maxN * h;
  const int64_t Nh = (int64_t)N * h;
  launch_ln_fwd<T>(c->st, xin, (const T*)P[0], (const T*)P[1], (T*)c->ln1,
                                                               c->ln1_m, c->ln1_r, N, h);
  if (c->use_lt & 1) {
    CB(lt_gemm(c, false, true, N, 3 * h, h, c->ln1, P[2], c->qkv, CUBLASLT_EPILOGUE_BIAS, P[3], nullptr));
  } else {
    (g_launches++, 0), bias_fill<T><<<grid_for(3 * Nh / 8), 256, 0, c->st>>>((T*)c->qkv, (const T*)P[3], 3 * h, 3 * Nh / 8);
    CB(rm_gemm(c, false, true, N, 3 * h, h, 1.f, c->ln1, dt, P[2], dt, 1.f, c->qkv, dt));
  }
  return 0;
}

template <class T>
int fwd_attn(gpt_ctx* c) {
  const int h = c->h, S = c->S, nh = c->nh, hd = h / nh, B = c->B;
  const cudaDataType_t dt = c->dt;
  const int BH = B * nh;
  const float scale = 1.0f / sqrtf((float)hd);
  CB(gemm_ptr(c, false, true, S, S, hd, scale, AP(c, PQ), dt, 3 * h, AP(c, PK), dt, 3 * h, 0.f, AP(c, PS),
              CUDA_R_32F, S, BH));
  int r = softmax<T>(c, (int64_t)BH * S, false);
  if (r) return r;
  CB(gemm_ptr(c, false, false, S, hd, S, 1.f, AP(c, PP), dt, S, AP(c, PV), dt, 3 * h, 0.f, AP(c, PO), dt, h, BH));
  return 0;
}

template <class T>
int fwd_out(gpt_ctx* c, int l, void* const* P, bool write_out) {
  const int N = c->N, h = c->h;
  const cudaDataType_t dt = c->dt;
  const float* xin = c->x + (int64_t)l * c->maxN * h;
  float* xout = c->x + (int64_t)(l + 1) * c->maxN * h;
  const int64_t Nh = (int64_t)N * h;
  (g_launches++, 0), resid_bias<T><<<grid_for(Nh / 8), 256, 0, c->st>>>(xin, (const T*)P[5], c->x_mid, h, Nh / 8);
  CB(rm_gemm(c, false, true, N, h, h, 1.f, c->att, dt, P[4], dt, 1.f, c->x_mid, CUDA_R_32F));
  launch_ln_fwd<T>(c->st, c->x_mid, (const T*)P[6], (const T*)P[7],
                                                               (T*)c->ln2, c->ln2_m, c->ln2_r, N, h);
  if (c->use_lt & 2) {
    CB(lt_gemm(c, false, true, N, 4 * h, h, c->ln2, P[8], c->fc_act, CUBLASLT_EPILOGUE_GELU_AUX_BIAS, P[9], c->fc_pre));
  } else {
    (g_launches++, 0), bias_fill<T><<<grid_for(4 * Nh / 8), 256, 0, c->st>>>((T*)c->fc_pre, (const T*)P[9], 4 * h,
                                                                            4 * Nh / 8);
    CB(rm_gemm(c, false, true, N, 4 * h, h, 1.f, c->ln2, dt, P[8], dt, 1.f, c->fc_pre, dt));
    (g_launches++, 0), gelu_fwd<T><<<grid_for(4 * Nh / 8), 256, 0, c->st>>>((const T*)c->fc_pre, (T*)c->fc_act,
                                                                           4 * Nh / 8);
  }
  if (write_out) {
    (g_launches++, 0), resid_bias<T><<<grid_for(Nh / 8), 256, 0, c->st>>>(c->x_mid, (const T*)P[11], xout, h, Nh / 8);
    CB(rm_gemm(c, false, true, N, h, 4 * h, 1.f, c->fc_act, dt, P[10], dt, 1.f, xout, CUDA_R_32F));
  }
  CK(cudaGetLastError());
  return 0;
}

template <class T>
int layer_fwd_impl(gpt_ctx* c, int l, void* const* P, bool write_out) {
  int r;
  if ((r = fwd_qkv<T>(c, l, P))) return r;
  if ((r = fwd_attn<T>(c))) return r;
  return fwd_out<T>(c, l, P, write_out);
}

// Block backward in three stages (after the forward of the layer was recomputed):
//   bwd_mlp:  MLP and W_o backward, LN2 backward; d_att = d(x_mid) W_o  -> c->datt [N, h]
//   bwd_attn: dq, dk, dv of the attention core (cuBLAS path)           -> c->dqkv [N, 3h]
//   bwd_qkv:  W_qkv backward, LN1 backward (residual gradient propagated in place)
template <class T>
int bwd_mlp(gpt_ctx* c, int l, void* const* P, float* const* G) {
  (void)l;
  const int N = c->N, h = c->h;
  const cudaDataType_t dt = c->dt;
  const int64_t Nh = (int64_t)N * h;
  int r;
  (g_launches++, 0), cast_f2t<T><<<grid_for(Nh / 8), 256, 0, c->st>>>(c->dres, (T*)c->dy, Nh / 8);
  CB(rm_gemm(c, true, false, h, 4 * h, N, 1.f, c->dy, dt, c->fc_act, dt, 0.f, G[10], CUDA_R_32F));
  if ((r = colsum(c, c->dres, true, N, h, G[11]))) return r;
  if (c->use_lt & 4) {
    CB(lt_gemm(c, false, false, N, 4 * h, h, c->dy, P[10], c->d4h, CUBLASLT_EPILOGUE_DGELU, nullptr, c->fc_pre));
  } else {
    CB(rm_gemm(c, false, false, N, 4 * h, h, 1.f, c->dy, dt, P[10], dt, 0.f, c->d4h, dt));
    (g_launches++, 0), gelu_bwd<T><<<grid_for(4 * Nh / 8), 256, 0, c->st>>>((T*)c->d4h, (const T*)c->fc_pre, 4 * Nh / 8);
  }
  CB(rm_gemm(c, true, false, 4 * h, h, N, 1.f, c->d4h, dt, c->ln2, dt, 0.f, G[8], CUDA_R_32F));
  if ((r = colsum(c, c->d4h, false, N, 4 * h, G[9]))) return r;
  CB(rm_gemm(c, false, false, N, h, 4 * h, 1.f, c->d4h, dt, P[8], dt, 0.f, c->dln, CUDA_R_32F));
  launch_ln_bwd<T>(c->st, c->dln, c->x_mid, c->ln2_m, c->ln2_r, (const T*)P[6],
                                                               c->dres, c->tmp, N, h);
  if ((r = colsum(c, c->tmp, true, N, h, G[6]))) return r;
  if ((r = colsum(c, c->dln, true, N, h, G[7]))) return r;
  (g_launches++, 0), cast_f2t<T><<<grid_for(Nh / 8), 256, 0, c->st>>>(c->dres, (T*)c->dy, Nh / 8);
  CB(rm_gemm(c, true, false, h, h, N, 1.f, c->dy, dt, c->att, dt, 0.f, G[4], CUDA_R_32F));
  if ((r = colsum(c, c->dres, true, N, h, G[5]))) return r;
  CB(rm_gemm(c, false, false, N, h, h, 1.f, c->dy, dt, P[4], dt, 0.f, c->datt, dt));
  return 0;
}

template <class T>
int bwd_attn(gpt_ctx* c) {
  const int h = c->h, S = c->S, nh = c->nh, hd = h / nh, B = c->B;
  const cudaDataType_t dt = c->dt;
  const int BH = B * nh;
  const float scale = 1.0f / sqrtf((float)hd);
  CB(gemm_ptr(c, false, true, S, S, hd, 1.f, AP(c, PDO), dt, h, AP(c, PV), dt, 3 * h, 0.f, AP(c, PS), CUDA_R_32F, S,
              BH));
  CB(gemm_ptr(c, true, false, S, hd, S, 1.f, AP(c, PP), dt, S, AP(c, PDO), dt, h, 0.f, AP(c, PDV), dt, 3 * h, BH));
  int r = softmax<T>(c, (int64_t)BH * S, true);
  if (r) return r;
  CB(gemm_ptr(c, false, false, S, hd, S, scale, AP(c, PP), dt, S, AP(c, PK), dt, 3 * h, 0.f, AP(c, PDQ), dt, 3 * h,
              BH));
  CB(gemm_ptr(c, true, false, S, hd, S, scale, AP(c, PP), dt, S, AP(c, PQ), dt, 3 * h, 0.f, AP(c, PDK), dt, 3 * h,
              BH));
  return 0;
}

template <class T>
int bwd_qkv(gpt_ctx* c, int l, void* const* P, float* const* G) {
  const int N = c->N, h = c->h;
  const cudaDataType_t dt = c->dt;
  const float* xin = c->x + (int64_t)l * c->maxN * h;
  int r;
  CB(rm_gemm(c, true, false, 3 * h, h, N, 1.f, c->dqkv, dt, c->ln1, dt, 0.f, G[2], CUDA_R_32F));
  if ((r = colsum(c, c->dqkv, false, N, 3 * h, G[3]))) return r;
  CB(rm_gemm(c, false, false, N, h, 3 * h, 1.f, c->dqkv, dt, P[2], dt, 0.f, c->dln, CUDA_R_32F));
  launch_ln_bwd<T>(c->st, c->dln, xin, c->ln1_m, c->ln1_r, (const T*)P[0],
                                                               c->dres, c->tmp, N, h);
  if ((r = colsum(c, c->tmp, true, N, h, G[0]))) return r;
  if ((r = colsum(c, c->dln, true, N, h, G[1]))) return r;
  CK(cudaGetLastError());
  return 0;
}

template <class T>
int layer_bwd_impl(gpt_ctx* c, int l, void* const* P, float* const* G) {
  int r = layer_fwd_impl<T>(c, l, P, false);  // recompute (activation checkpointing)
  if (r) return r;
  if ((r = bwd_mlp<T>(c, l, P, G))) return r;
  if ((r = bwd_attn<T>(c))) return r;
  return bwd_qkv<T>(c, l, P, G);
}

template <class T>
int head_impl(gpt_ctx* c, const int* tok, void* const* R, float* const* G, float* d_loss, bool backward = true) {
  const int N = c->N, h = c->h, V = c->V, S = c->S;
  const cudaDataType_t dt = c->dt;
  const float* xL = c->x + (int64_t)c->L * c->maxN * h;
  launch_ln_fwd<T>(c->st, xL, (const T*)R[2], (const T*)R[3], (T*)c->lnf,
                                                               c->lnf_m, c->lnf_r, N, h);
  CB(rm_gemm(c, false, true, N, V, h, 1.f, c->lnf, dt, R[0], dt, 0.f, c->logits, CUDA_R_32F));
  (g_launches++, 0), ce_fwd_bwd<T><<<N, 512, 0, c->st>>>(c->logits, tok, S, V, 1.0f / N, c->row_loss, (T*)c->dlogits);
  (g_launches++, 0), mean_fixed<<<1, 512, 0, c->st>>>(c->row_loss, N, 1.0f / N, d_loss);
  if (!backward) {
    CK(cudaGetLastError());
    return 0;
  }
  CB(rm_gemm(c, false, false, N, h, V, 1.f, c->dlogits, dt, R[0], dt, 0.f, c->dln, CUDA_R_32F));
  CK(cudaMemsetAsync(c->dres, 0, sizeof(float) * (size_t)N * h, c->st));
  launch_ln_bwd<T>(c->st, c->dln, xL, c->lnf_m, c->lnf_r, (const T*)R[2], c->dres,
                                                               c->tmp, N, h);
  int r;
  if ((r = colsum(c, c->tmp, true, N, h, G[2]))) return r;
  if ((r = colsum(c, c->dln, true, N, h, G[3]))) return r;
  CB(rm_gemm(c, true, false, V, h, N, 1.f, c->dlogits, dt, c->lnf, dt, 0.f, G[0], CUDA_R_32F));
  CK(cudaGetLastError());
  return 0;
}

}  // namespace

extern "C" {

const char* gpt_last_error(void) { return g_err.c_str(); }
int64_t gpt_kernel_launches(void) { return g_launches.load(); }
int64_t gpt_workspace_bytes(const gpt_ctx* c) { return c ? c->bytes : 0; }
float* gpt_checkpoint(gpt_ctx* c, int32_t l) {
  if (!c || l < 0 || l > c->L) return nullptr;
  return c->x + (int64_t)l * c->maxN * c->h;
}

int32_t gpt_create(const gpt_config* cfg, gpt_ctx** out) {
  g_err.clear();
  if (!cfg || !out || cfg->n_layers < 1 || cfg->hidden < 8 || cfg->heads < 1 || cfg->hidden % cfg->heads ||
      cfg->hidden % 8 || (cfg->hidden / cfg->heads) % 8 || cfg->seq < 8 || cfg->seq % 8 || cfg->max_batch < 1 ||
      cfg->vocab < 8 || cfg->vocab % 8 || !cfg->stream) {
    seterr("gpt_create: invalid config (hidden, head dim, seq and vocab must be multiples of 8; stream required)");
    return -1;
  }
  const int nch = (cfg->seq / 8 + 31) / 32;
  if (nch != 1 && nch != 2 && nch != 4 && nch != 8) {
    seterr("gpt_create: seq %d unsupported by the softmax kernel", cfg->seq);
    return -1;
  }
  auto* c = new gpt_ctx();
  c->cfg = *cfg;
  c->bf16 = cfg->precision == 1;
  c->es = c->bf16 ? 2 : 4;
  c->dt = c->bf16 ? CUDA_R_16BF : CUDA_R_32F;
  c->st = static_cast<cudaStream_t>(cfg->stream);
  c->S = cfg->seq;
  c->h = cfg->hidden;
  c->nh = cfg->heads;
  c->V = cfg->vocab;
  c->L = cfg->n_layers;
  c->maxN = (int64_t)cfg->max_batch * cfg->seq;
  const int64_t mN = c->maxN, h = c->h, es = c->es;
  const int64_t BHSS = (int64_t)cfg->max_batch * c->nh * c->S * c->S;
  int r = 0;
  if (cudaSetDevice(cfg->device) != cudaSuccess) {
    seterr("gpt_create: cudaSetDevice failed");
    delete c;
    return -2;
  }
  auto A = [&](void** p, int64_t b) {
    if (!r) r = alloc(c, p, b);
  };
  A((void**)&c->x, 4 * (c->L + 1) * mN * h);
  for (void** p : {&c->ln1, &c->ln2, &c->lnf, &c->att, &c->dy, &c->datt}) A(p, es * mN * h);
  for (void** p : {&c->qkv, &c->dqkv}) A(p, es * mN * 3 * h);
  for (void** p : {&c->fc_pre, &c->fc_act, &c->d4h}) A(p, es * mN * 4 * h);
  A(&c->probs, es * BHSS);
  A((void**)&c->scores, 4 * BHSS);
  for (float** p : {&c->ln1_m, &c->ln1_r, &c->ln2_m, &c->ln2_r, &c->lnf_m, &c->lnf_r, &c->row_loss, &c->ones_f})
    A((void**)p, 4 * mN);
  for (float** p : {&c->x_mid, &c->dres, &c->dln, &c->tmp}) A((void**)p, 4 * mN * h);
  A((void**)&c->logits, 4 * mN * c->V);
  if (c->bf16)
    A(&c->dlogits, 2 * mN * c->V);
  else
    c->dlogits = c->logits;  // fp32: dlogits overwrite logits in place
  A(&c->ones_t, es * mN);
  A((void**)&c->aptr, 10 * 8 * (int64_t)cfg->max_batch * c->nh);
  for (int** p : {&c->keys, &c->vals, &c->keys2, &c->vals2}) A((void**)p, 4 * mN);
  A(&c->ws, c->ws_bytes);
  if (!r) {
    cub::DeviceRadixSort::SortPairs(nullptr, c->cub_bytes, c->keys, c->keys2, c->vals, c->vals2, (int)mN);
    A(&c->cub_tmp, c->cub_bytes + 256);
  }
  if (r) {
    gpt_destroy(c);
    return r;
  }
  if (cublasCreate(&c->cb) != CUBLAS_STATUS_SUCCESS) {
    seterr("gpt_create: cublasCreate failed");
    gpt_destroy(c);
    return -4;
  }
  cublasSetStream(c->cb, c->st);
  cublasSetWorkspace(c->cb, c->ws, c->ws_bytes);
  cublasSetMathMode(c->cb, CUBLAS_DEFAULT_MATH);  // no TF32 in fp32 mode
  cublasSetAtomicsMode(c->cb, CUBLAS_ATOMICS_NOT_ALLOWED);
  if (c->bf16) {
    const char* e = getenv("SH_GPT_LT");
    const int mask = e ? atoi(e) : 7;
    c->use_lt = mask != 0 && cublasLtCreate(&c->lt) == CUBLAS_STATUS_SUCCESS ? mask : 0;
  }
  (g_launches++, 0), fill_ones<float><<<grid_for(mN), 256, 0, c->st>>>(c->ones_f, mN);
  if (c->bf16)
    (g_launches++, 0), fill_ones<bf16><<<grid_for(mN), 256, 0, c->st>>>((bf16*)c->ones_t, mN);
  else
    (g_launches++, 0), fill_ones<float><<<grid_for(mN), 256, 0, c->st>>>((float*)c->ones_t, mN);
  if (cudaStreamSynchronize(c->st) != cudaSuccess) {
    seterr("gpt_create: init kernels failed");
    gpt_destroy(c);
    return -2;
  }
  *out = c;
  return 0;
}

int32_t gpt_destroy(gpt_ctx* c) {
  if (!c) return 0;
  if (c->st) cudaStreamSynchronize(c->st);
  if (c->cb) cublasDestroy(c->cb);
  if (c->lt) cublasLtDestroy(c->lt);
  for (void* p : c->allocs) cudaFree(p);
  delete c;
  return 0;
}

int32_t gpt_embed_forward(gpt_ctx* c, const int32_t* tok, int32_t B, void* const* R) {
  g_err.clear();
  if (!c || !tok || !R || B < 1 || (int64_t)B * c->S > c->maxN) {
    seterr("gpt_embed_forward: bad batch %d", B);
    return -1;
  }
  c->B = B;
  c->N = B * c->S;
  if (c->ptrB != B) {
    const int BH = B * c->nh;
    (g_launches++, 0), build_attn_ptrs<<<(BH + 127) / 128, 128, 0, c->st>>>(
        c->aptr, (char*)c->qkv, (char*)c->scores, (char*)c->probs, (char*)c->att, (char*)c->datt, (char*)c->dqkv, B,
        c->nh, c->S, c->h, c->es);
    c->ptrB = B;
  }
  if (c->bf16)
    (g_launches++, 0), embed_fwd<bf16><<<c->N, 128, 0, c->st>>>(tok, (const bf16*)R[0], (const bf16*)R[1], c->x, c->S, c->h);
  else
    (g_launches++, 0), embed_fwd<float><<<c->N, 128, 0, c->st>>>(tok, (const float*)R[0], (const float*)R[1], c->x, c->S, c->h);
  CK(cudaGetLastError());
  return 0;
}

int32_t gpt_layer_forward(gpt_ctx* c, int32_t l, void* const* P) {
  g_err.clear();
  if (!c || !P || l < 0 || l >= c->L || c->B == 0) {
    seterr("gpt_layer_forward: bad layer %d or no embed_forward", l);
    return -1;
  }
  return c->bf16 ? layer_fwd_impl<bf16>(c, l, P, true) : layer_fwd_impl<float>(c, l, P, true);
}

int32_t gpt_head_forward_backward(gpt_ctx* c, const int32_t* tok, void* const* R, float* const* G, float* d_loss) {
  g_err.clear();
  if (!c || !tok || !R || !G || !d_loss || c->B == 0) {
    seterr("gpt_head_forward_backward: bad arguments");
    return -1;
  }
  return c->bf16 ? head_impl<bf16>(c, tok, R, G, d_loss) : head_impl<float>(c, tok, R, G, d_loss);
}

int32_t gpt_head_forward(gpt_ctx* c, const int32_t* tok, void* const* R, float* d_loss) {
  g_err.clear();
  if (!c || !tok || !R || !d_loss || c->B == 0) {
    seterr("gpt_head_forward: bad arguments");
    return -1;
  }
  return c->bf16 ? head_impl<bf16>(c, tok, R, nullptr, d_loss, false)
                 : head_impl<float>(c, tok, R, nullptr, d_loss, false);
}

int32_t gpt_layer_backward(gpt_ctx* c, int32_t l, void* const* P, float* const* G) {
  g_err.clear();
  if (!c || !P || !G || l < 0 || l >= c->L || c->B == 0) {
    seterr("gpt_layer_backward: bad layer %d", l);
    return -1;
  }
  return c->bf16 ? layer_bwd_impl<bf16>(c, l, P, G) : layer_bwd_impl<float>(c, l, P, G);
}

static bool stage_ok(gpt_ctx* c, int32_t l, const void* P) {
  if (!c || !P || l < 0 || l >= c->L || c->B == 0) {
    seterr("gpt stage: bad layer %d or no embed_forward", l);
    return false;
  }
  return true;
}

int32_t gpt_layer_forward_qkv(gpt_ctx* c, int32_t l, void* const* P) {
  g_err.clear();
  if (!stage_ok(c, l, P)) return -1;
  return c->bf16 ? fwd_qkv<bf16>(c, l, P) : fwd_qkv<float>(c, l, P);
}

int32_t gpt_layer_forward_out(gpt_ctx* c, int32_t l, void* const* P, int32_t write_out) {
  g_err.clear();
  if (!stage_ok(c, l, P)) return -1;
  return c->bf16 ? fwd_out<bf16>(c, l, P, write_out != 0) : fwd_out<float>(c, l, P, write_out != 0);
}

int32_t gpt_layer_backward_mlp(gpt_ctx* c, int32_t l, void* const* P, float* const* G) {
  g_err.clear();
  if (!stage_ok(c, l, P) || !G) return -1;
  return c->bf16 ? bwd_mlp<bf16>(c, l, P, G) : bwd_mlp<float>(c, l, P, G);
}

int32_t gpt_layer_backward_qkv(gpt_ctx* c, int32_t l, void* const* P, float* const* G) {
  g_err.clear();
  if (!stage_ok(c, l, P) || !G) return -1;
  return c->bf16 ? bwd_qkv<bf16>(c, l, P, G) : bwd_qkv<float>(c, l, P, G);
}

void* gpt_buffer(gpt_ctx* c, int32_t which) {
  if (!c) return nullptr;
  switch (which) {
    case 0: return c->qkv;
    case 1: return c->att;
    case 2: return c->datt;
    case 3: return c->dqkv;
    default: return nullptr;
  }
}

int32_t gpt_embed_backward(gpt_ctx* c, const int32_t* tok, float* const* G) {
  g_err.clear();
  if (!c || !tok || !G || c->B == 0) {
    seterr("gpt_embed_backward: bad arguments");
    return -1;
  }
  const int N = c->N;
  (g_launches++, 0), gather_tokens<<<(N + 255) / 256, 256, 0, c->st>>>(tok, c->S, N, c->keys, c->vals);
  int bits = 1;
  while ((1 << bits) < c->V) ++bits;
  size_t tb = c->cub_bytes;
  CK(cub::DeviceRadixSort::SortPairs(c->cub_tmp, tb, c->keys, c->keys2, c->vals, c->vals2, N, 0, bits, c->st));
  (g_launches++, 0), embed_bwd_wte<<<N, 256, 0, c->st>>>(c->keys2, c->vals2, c->dres, G[0], N, c->h);
  (g_launches++, 0), embed_bwd_wpe<<<c->S, 256, 0, c->st>>>(c->dres, G[1], c->B, c->S, c->h);
  CK(cudaGetLastError());
  return 0;
}

}  // extern "C"
