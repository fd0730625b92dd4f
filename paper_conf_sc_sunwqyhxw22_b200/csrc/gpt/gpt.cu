// GPT-2 block compute that drives the offload engine -- OUTSIDE THE HOT PATH (see sh_gpt.h).
//
// GEMMs: cuBLAS (bf16 or fp32 operands, fp32 accumulation, CUBLAS_COMPUTE_32F, fixed
// workspace => run-to-run bitwise reproducible; on sm_100 the bf16 GEMMs run on tcgen05 tensor
// cores inside cuBLAS).  Everything else is small SIMT kernels with fixed reduction orders.
// The math is DESIGN.md reading R1 / oracle/gpt_oracle.py (shared by definition, not code).
#include <cublas_v2.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>

#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
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
  return r;  // every thread of warp 0.. holds the result (all warps compute it)
}

// ------------------------------------------------------------------------------ kernels
template <class T>
__global__ void embed_fwd(const int* tok, const T* wte, const T* wpe, float* x, int S, int h) {
  const int n = blockIdx.x;  // token row b*S+s
  const int b = n / S, s = n % S;
  const int t = tok[b * (S + 1) + s];
  for (int c = threadIdx.x; c < h; c += blockDim.x)
    x[(int64_t)n * h + c] = tof(wte[(int64_t)t * h + c]) + tof(wpe[(int64_t)s * h + c]);
}

template <class T>
__global__ void ln_fwd(const float* x, const T* g, const T* b, T* out, float* mean, float* rstd, int N, int h) {
  const int row = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= N) return;
  const float* xr = x + (int64_t)row * h;
  float s = 0.f;
  for (int c = lane; c < h; c += 32) s += xr[c];
  const float mu = warp_sum(s) / h;
  float v = 0.f;
  for (int c = lane; c < h; c += 32) {
    const float d = xr[c] - mu;
    v += d * d;
  }
  const float rs = 1.0f / sqrtf(warp_sum(v) / h + kLnEps);
  T* o = out + (int64_t)row * h;
  for (int c = lane; c < h; c += 32) o[c] = fromf<T>((xr[c] - mu) * rs * tof(g[c]) + tof(b[c]));
  if (lane == 0) {
    mean[row] = mu;
    rstd[row] = rs;
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
  for (int c = lane; c < h; c += 32) {
    const float xh = (xr[c] - mu) * rs;
    const float dxh = dr[c] * tof(g[c]);
    a += dxh;
    bb += dxh * xh;
  }
  a = warp_sum(a) / h;
  bb = warp_sum(bb) / h;
  float* o = dres + (int64_t)row * h;
  float* t = tmp + (int64_t)row * h;
  for (int c = lane; c < h; c += 32) {
    const float xh = (xr[c] - mu) * rs;
    const float dxh = dr[c] * tof(g[c]);
    o[c] += rs * (dxh - a - xh * bb);
    t[c] = dr[c] * xh;
  }
}

// qkv (fp32, no bias) [N,3h] + bias -> q,k,v [B,nh,S,hd] in T
template <class T>
__global__ void qkv_split(const float* qkv, const T* bias, T* q, T* k, T* v, int S, int h, int nh, int64_t total) {
  const int hd = h / nh;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = i / (3 * h);
    const int c = (int)(i % (3 * h));
    const int which = c / h, cc = c % h, head = cc / hd, d = cc % hd;
    const int64_t b = n / S, s = n % S;
    const int64_t dst = ((b * nh + head) * S + s) * hd + d;
    const T val = fromf<T>(qkv[i] + tof(bias[c]));
    (which == 0 ? q : which == 1 ? k : v)[dst] = val;
  }
}

// [B,nh,S,hd] <-> [N,h]
template <class T>
__global__ void heads_to_rows(const T* src, T* dst, int S, int h, int nh, int64_t total, int rows_stride, int col_off) {
  const int hd = h / nh;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = i / h;
    const int c = (int)(i % h), head = c / hd, d = c % hd;
    const int64_t b = n / S, s = n % S;
    dst[n * rows_stride + col_off + c] = src[((b * nh + head) * S + s) * hd + d];
  }
}
template <class T>
__global__ void rows_to_heads(const T* src, T* dst, int S, int h, int nh, int64_t total) {
  const int hd = h / nh;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = i / h;
    const int c = (int)(i % h), head = c / hd, d = c % hd;
    const int64_t b = n / S, s = n % S;
    dst[((b * nh + head) * S + s) * hd + d] = src[i];
  }
}

// causal softmax, one warp per row: scores already scaled by 1/sqrt(hd)
template <class T>
__global__ void softmax_causal(const float* sc, T* p, int S, int64_t rows) {
  const int64_t row = blockIdx.x * (int64_t)(blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= rows) return;
  const int r = (int)(row % S);
  const float* s = sc + row * S;
  T* o = p + row * S;
  float m = -INFINITY;
  for (int c = lane; c <= r; c += 32) m = fmaxf(m, s[c]);
  m = warp_max(m);
  float z = 0.f;
  for (int c = lane; c <= r; c += 32) z += expf(s[c] - m);
  z = warp_sum(z);
  const float inv = 1.0f / z;
  for (int c = lane; c < S; c += 32) o[c] = fromf<T>(c <= r ? expf(s[c] - m) * inv : 0.f);
}

// dS = P * (dP - Σ dP*P), written in place over P
template <class T>
__global__ void softmax_bwd(T* p, const float* dp, int S, int64_t rows) {
  const int64_t row = blockIdx.x * (int64_t)(blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= rows) return;
  const int r = (int)(row % S);
  T* pr = p + row * S;
  const float* d = dp + row * S;
  float a = 0.f;
  for (int c = lane; c <= r; c += 32) a += tof(pr[c]) * d[c];
  a = warp_sum(a);
  for (int c = lane; c <= r; c += 32) pr[c] = fromf<T>(tof(pr[c]) * (d[c] - a));
}

template <class T>
__global__ void resid_bias(const float* x, const T* b, float* out, int h, int64_t total) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = x[i] + tof(b[i % h]);
}

__device__ __forceinline__ float gelu_f(float u) {
  const float k = 0.7978845608028654f;  // sqrt(2/pi)
  return 0.5f * u * (1.0f + tanhf(k * (u + 0.044715f * u * u * u)));
}
__device__ __forceinline__ float gelu_grad(float u) {
  const float k = 0.7978845608028654f;
  const float t = tanhf(k * (u + 0.044715f * u * u * u));
  return 0.5f * (1.0f + t) + 0.5f * u * (1.0f - t * t) * k * (1.0f + 3.0f * 0.044715f * u * u);
}

template <class T>
__global__ void gelu_fwd(const float* f, const T* b, T* pre, T* act, int C, int64_t total) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const T u = fromf<T>(f[i] + tof(b[i % C]));
    pre[i] = u;
    act[i] = fromf<T>(gelu_f(tof(u)));
  }
}
template <class T>
__global__ void gelu_bwd(T* d, const T* pre, int64_t total) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
    d[i] = fromf<T>(tof(d[i]) * gelu_grad(tof(pre[i])));
}
template <class T>
__global__ void cast_f2t(const float* a, T* o, int64_t total) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
    o[i] = fromf<T>(a[i]);
}
template <class T>
__global__ void fill_ones(T* o, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    o[i] = fromf<T>(1.0f);
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
  for (int c = threadIdx.x; c < V; c += 512) m = fmaxf(m, l[c]);
  m = block_reduce<512>(m, true);
  float z = 0.f;
  for (int c = threadIdx.x; c < V; c += 512) z += expf(l[c] - m);
  z = block_reduce<512>(z, false);
  const float inv = 1.0f / z;
  const float lt = l[tgt];
  __syncthreads();  // all reads of l[] done before an in-place (fp32) overwrite
  T* d = dlogits + n * V;
  for (int c = threadIdx.x; c < V; c += 512) {
    float p = expf(l[c] - m) * inv;
    if (c == tgt) p -= 1.0f;
    d[c] = fromf<T>(p * inv_n);
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

int grid_for(int64_t total, int threads = 256) {
  int64_t g = (total + threads - 1) / threads;
  const int64_t cap = 148 * 16;
  return (int)(g < cap ? (g > 0 ? g : 1) : cap);
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
  int64_t maxN = 0;
  std::vector<void*> allocs;
  int64_t bytes = 0;
  float* x = nullptr;  // (L+1) checkpoints
  void *ln1, *ln2, *lnf, *q, *k, *v, *probs, *atto, *att, *fc_pre, *fc_act, *dy, *d4h, *datt, *dO, *dq, *dk, *dv, *dqkv, *ones_t, *dlogits;
  float *ln1_m, *ln1_r, *ln2_m, *ln2_r, *lnf_m, *lnf_r, *f32big, *scores, *x_mid, *dres, *dln, *tmp, *logits, *row_loss, *ones_f;
  int *keys, *vals, *keys2, *vals2;
  void* cub_tmp = nullptr;
  size_t cub_bytes = 0;
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

// Row-major C[M,N] = alpha op(A) op(B) + beta C.  A is [M,K] (or stored [K,M] if tA),
// B is [K,N] (or stored [N,K] if tB).  Column-major cuBLAS computes C^T = op(B)^T op(A)^T.
cublasStatus_t rm_gemm(gpt_ctx* c, bool tA, bool tB, int M, int N, int K, float alpha, const void* A,
                       cudaDataType_t ta, const void* B, cudaDataType_t tb, float beta, void* C, cudaDataType_t tc) {
  const int lda = tA ? M : K, ldb = tB ? K : N;
  return cublasGemmEx(c->cb, tB ? CUBLAS_OP_T : CUBLAS_OP_N, tA ? CUBLAS_OP_T : CUBLAS_OP_N, N, M, K, &alpha, B, tb,
                      ldb, A, ta, lda, &beta, C, tc, N, CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
}
cublasStatus_t rm_gemm_batched(gpt_ctx* c, bool tA, bool tB, int M, int N, int K, float alpha, const void* A,
                               cudaDataType_t ta, int64_t sA, const void* B, cudaDataType_t tb, int64_t sB, float beta,
                               void* C, cudaDataType_t tc, int64_t sC, int batch) {
  const int lda = tA ? M : K, ldb = tB ? K : N;
  return cublasGemmStridedBatchedEx(c->cb, tB ? CUBLAS_OP_T : CUBLAS_OP_N, tA ? CUBLAS_OP_T : CUBLAS_OP_N, N, M, K,
                                    &alpha, B, tb, ldb, sB, A, ta, lda, sA, &beta, C, tc, N, sC, batch,
                                    CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
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

template <class T>
int layer_fwd_impl(gpt_ctx* c, int l, void* const* P, bool write_out) {
  const int N = c->N, h = c->h, S = c->S, nh = c->nh, hd = h / nh, B = c->B;
  const cudaDataType_t dt = c->dt;
  const float* xin = c->x + (int64_t)l * c->maxN * h;
  float* xout = c->x + (int64_t)(l + 1) * c->maxN * h;
  const int rows_per_blk = 8;
  (g_launches++, 0), ln_fwd<T><<<(N + rows_per_blk - 1) / rows_per_blk, 256, 0, c->st>>>(xin, (const T*)P[0], (const T*)P[1], (T*)c->ln1,
                                                                      c->ln1_m, c->ln1_r, N, h);
  CB(rm_gemm(c, false, true, N, 3 * h, h, 1.f, c->ln1, dt, P[2], dt, 0.f, c->f32big, CUDA_R_32F));
  (g_launches++, 0), qkv_split<T><<<grid_for((int64_t)N * 3 * h), 256, 0, c->st>>>(c->f32big, (const T*)P[3], (T*)c->q, (T*)c->k,
                                                                (T*)c->v, S, h, nh, (int64_t)N * 3 * h);
  const int BH = B * nh;
  const float scale = 1.0f / sqrtf((float)hd);
  CB(rm_gemm_batched(c, false, true, S, S, hd, scale, c->q, dt, (int64_t)S * hd, c->k, dt, (int64_t)S * hd, 0.f,
                     c->scores, CUDA_R_32F, (int64_t)S * S, BH));
  const int64_t rows = (int64_t)BH * S;
  (g_launches++, 0), softmax_causal<T><<<(int)((rows + 7) / 8), 256, 0, c->st>>>(c->scores, (T*)c->probs, S, rows);
  CB(rm_gemm_batched(c, false, false, S, hd, S, 1.f, c->probs, dt, (int64_t)S * S, c->v, dt, (int64_t)S * hd, 0.f,
                     c->atto, dt, (int64_t)S * hd, BH));
  (g_launches++, 0), heads_to_rows<T><<<grid_for((int64_t)N * h), 256, 0, c->st>>>((const T*)c->atto, (T*)c->att, S, h, nh,
                                                                 (int64_t)N * h, h, 0);
  (g_launches++, 0), resid_bias<T><<<grid_for((int64_t)N * h), 256, 0, c->st>>>(xin, (const T*)P[5], c->x_mid, h, (int64_t)N * h);
  CB(rm_gemm(c, false, true, N, h, h, 1.f, c->att, dt, P[4], dt, 1.f, c->x_mid, CUDA_R_32F));
  (g_launches++, 0), ln_fwd<T><<<(N + rows_per_blk - 1) / rows_per_blk, 256, 0, c->st>>>(c->x_mid, (const T*)P[6], (const T*)P[7],
                                                                      (T*)c->ln2, c->ln2_m, c->ln2_r, N, h);
  CB(rm_gemm(c, false, true, N, 4 * h, h, 1.f, c->ln2, dt, P[8], dt, 0.f, c->f32big, CUDA_R_32F));
  (g_launches++, 0), gelu_fwd<T><<<grid_for((int64_t)N * 4 * h), 256, 0, c->st>>>(c->f32big, (const T*)P[9], (T*)c->fc_pre,
                                                               (T*)c->fc_act, 4 * h, (int64_t)N * 4 * h);
  if (write_out) {
    (g_launches++, 0), resid_bias<T><<<grid_for((int64_t)N * h), 256, 0, c->st>>>(c->x_mid, (const T*)P[11], xout, h, (int64_t)N * h);
    CB(rm_gemm(c, false, true, N, h, 4 * h, 1.f, c->fc_act, dt, P[10], dt, 1.f, xout, CUDA_R_32F));
  }
  CK(cudaGetLastError());
  return 0;
}

template <class T>
int layer_bwd_impl(gpt_ctx* c, int l, void* const* P, float* const* G) {
  int r = layer_fwd_impl<T>(c, l, P, false);  // recompute (activation checkpointing)
  if (r) return r;
  const int N = c->N, h = c->h, S = c->S, nh = c->nh, hd = h / nh, B = c->B;
  const cudaDataType_t dt = c->dt;
  const float* xin = c->x + (int64_t)l * c->maxN * h;
  const int64_t Nh = (int64_t)N * h;
  // ---- MLP
  (g_launches++, 0), cast_f2t<T><<<grid_for(Nh), 256, 0, c->st>>>(c->dres, (T*)c->dy, Nh);
  CB(rm_gemm(c, true, false, h, 4 * h, N, 1.f, c->dy, dt, c->fc_act, dt, 0.f, G[10], CUDA_R_32F));
  if ((r = colsum(c, c->dres, true, N, h, G[11]))) return r;
  CB(rm_gemm(c, false, false, N, 4 * h, h, 1.f, c->dy, dt, P[10], dt, 0.f, c->d4h, dt));
  (g_launches++, 0), gelu_bwd<T><<<grid_for(4 * Nh), 256, 0, c->st>>>((T*)c->d4h, (const T*)c->fc_pre, 4 * Nh);
  CB(rm_gemm(c, true, false, 4 * h, h, N, 1.f, c->d4h, dt, c->ln2, dt, 0.f, G[8], CUDA_R_32F));
  if ((r = colsum(c, c->d4h, false, N, 4 * h, G[9]))) return r;
  CB(rm_gemm(c, false, false, N, h, 4 * h, 1.f, c->d4h, dt, P[8], dt, 0.f, c->dln, CUDA_R_32F));
  (g_launches++, 0), ln_bwd<T><<<(N + 7) / 8, 256, 0, c->st>>>(c->dln, c->x_mid, c->ln2_m, c->ln2_r, (const T*)P[6], c->dres, c->tmp, N, h);
  if ((r = colsum(c, c->tmp, true, N, h, G[6]))) return r;
  if ((r = colsum(c, c->dln, true, N, h, G[7]))) return r;
  // ---- attention
  (g_launches++, 0), cast_f2t<T><<<grid_for(Nh), 256, 0, c->st>>>(c->dres, (T*)c->dy, Nh);
  CB(rm_gemm(c, true, false, h, h, N, 1.f, c->dy, dt, c->att, dt, 0.f, G[4], CUDA_R_32F));
  if ((r = colsum(c, c->dres, true, N, h, G[5]))) return r;
  CB(rm_gemm(c, false, false, N, h, h, 1.f, c->dy, dt, P[4], dt, 0.f, c->datt, dt));
  (g_launches++, 0), rows_to_heads<T><<<grid_for(Nh), 256, 0, c->st>>>((const T*)c->datt, (T*)c->dO, S, h, nh, Nh);
  const int BH = B * nh;
  const float scale = 1.0f / sqrtf((float)hd);
  const int64_t sQ = (int64_t)S * hd, sS = (int64_t)S * S;
  CB(rm_gemm_batched(c, false, true, S, S, hd, 1.f, c->dO, dt, sQ, c->v, dt, sQ, 0.f, c->scores, CUDA_R_32F, sS, BH));
  CB(rm_gemm_batched(c, true, false, S, hd, S, 1.f, c->probs, dt, sS, c->dO, dt, sQ, 0.f, c->dv, dt, sQ, BH));
  const int64_t rows = (int64_t)BH * S;
  (g_launches++, 0), softmax_bwd<T><<<(int)((rows + 7) / 8), 256, 0, c->st>>>((T*)c->probs, c->scores, S, rows);
  CB(rm_gemm_batched(c, false, false, S, hd, S, scale, c->probs, dt, sS, c->k, dt, sQ, 0.f, c->dq, dt, sQ, BH));
  CB(rm_gemm_batched(c, true, false, S, hd, S, scale, c->probs, dt, sS, c->q, dt, sQ, 0.f, c->dk, dt, sQ, BH));
  (g_launches++, 0), heads_to_rows<T><<<grid_for(Nh), 256, 0, c->st>>>((const T*)c->dq, (T*)c->dqkv, S, h, nh, Nh, 3 * h, 0);
  (g_launches++, 0), heads_to_rows<T><<<grid_for(Nh), 256, 0, c->st>>>((const T*)c->dk, (T*)c->dqkv, S, h, nh, Nh, 3 * h, h);
  (g_launches++, 0), heads_to_rows<T><<<grid_for(Nh), 256, 0, c->st>>>((const T*)c->dv, (T*)c->dqkv, S, h, nh, Nh, 3 * h, 2 * h);
  CB(rm_gemm(c, true, false, 3 * h, h, N, 1.f, c->dqkv, dt, c->ln1, dt, 0.f, G[2], CUDA_R_32F));
  if ((r = colsum(c, c->dqkv, false, N, 3 * h, G[3]))) return r;
  CB(rm_gemm(c, false, false, N, h, 3 * h, 1.f, c->dqkv, dt, P[2], dt, 0.f, c->dln, CUDA_R_32F));
  (g_launches++, 0), ln_bwd<T><<<(N + 7) / 8, 256, 0, c->st>>>(c->dln, xin, c->ln1_m, c->ln1_r, (const T*)P[0], c->dres, c->tmp, N, h);
  if ((r = colsum(c, c->tmp, true, N, h, G[0]))) return r;
  if ((r = colsum(c, c->dln, true, N, h, G[1]))) return r;
  CK(cudaGetLastError());
  return 0;
}

template <class T>
int head_impl(gpt_ctx* c, const int* tok, void* const* R, float* const* G, float* d_loss) {
  const int N = c->N, h = c->h, V = c->V, S = c->S;
  const cudaDataType_t dt = c->dt;
  const float* xL = c->x + (int64_t)c->L * c->maxN * h;
  (g_launches++, 0), ln_fwd<T><<<(N + 7) / 8, 256, 0, c->st>>>(xL, (const T*)R[2], (const T*)R[3], (T*)c->lnf, c->lnf_m, c->lnf_r, N, h);
  CB(rm_gemm(c, false, true, N, V, h, 1.f, c->lnf, dt, R[0], dt, 0.f, c->logits, CUDA_R_32F));
  (g_launches++, 0), ce_fwd_bwd<T><<<N, 512, 0, c->st>>>(c->logits, tok, S, V, 1.0f / N, c->row_loss, (T*)c->dlogits);
  (g_launches++, 0), mean_fixed<<<1, 512, 0, c->st>>>(c->row_loss, N, 1.0f / N, d_loss);
  CB(rm_gemm(c, false, false, N, h, V, 1.f, c->dlogits, dt, R[0], dt, 0.f, c->dln, CUDA_R_32F));
  CK(cudaMemsetAsync(c->dres, 0, sizeof(float) * (size_t)N * h, c->st));
  (g_launches++, 0), ln_bwd<T><<<(N + 7) / 8, 256, 0, c->st>>>(c->dln, xL, c->lnf_m, c->lnf_r, (const T*)R[2], c->dres, c->tmp, N, h);
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
  if (!cfg || !out || cfg->n_layers < 1 || cfg->hidden < 1 || cfg->heads < 1 || cfg->hidden % cfg->heads ||
      cfg->seq < 1 || cfg->max_batch < 1 || cfg->vocab < 1 || !cfg->stream) {
    seterr("gpt_create: invalid config (hidden %% heads must be 0, stream required)");
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
  for (void** p : {&c->ln1, &c->ln2, &c->lnf, &c->q, &c->k, &c->v, &c->atto, &c->att, &c->dy, &c->datt, &c->dO, &c->dq,
                   &c->dk, &c->dv})
    A(p, es * mN * h);
  A(&c->dqkv, es * mN * 3 * h);
  for (void** p : {&c->fc_pre, &c->fc_act, &c->d4h}) A(p, es * mN * 4 * h);
  A(&c->probs, es * BHSS);
  A((void**)&c->scores, 4 * BHSS);
  for (float** p : {&c->ln1_m, &c->ln1_r, &c->ln2_m, &c->ln2_r, &c->lnf_m, &c->lnf_r, &c->row_loss, &c->ones_f})
    A((void**)p, 4 * mN);
  A((void**)&c->f32big, 4 * mN * 4 * h);
  for (float** p : {&c->x_mid, &c->dres, &c->dln, &c->tmp}) A((void**)p, 4 * mN * h);
  A((void**)&c->logits, 4 * mN * c->V);
  if (c->bf16)
    A(&c->dlogits, 2 * mN * c->V);
  else
    c->dlogits = c->logits;  // fp32: dlogits overwrite logits in place
  A(&c->ones_t, es * mN);
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
  if (c->bf16)
    (g_launches++, 0), embed_fwd<bf16><<<c->N, 256, 0, c->st>>>(tok, (const bf16*)R[0], (const bf16*)R[1], c->x, c->S, c->h);
  else
    (g_launches++, 0), embed_fwd<float><<<c->N, 256, 0, c->st>>>(tok, (const float*)R[0], (const float*)R[1], c->x, c->S, c->h);
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

int32_t gpt_layer_backward(gpt_ctx* c, int32_t l, void* const* P, float* const* G) {
  g_err.clear();
  if (!c || !P || !G || l < 0 || l >= c->L || c->B == 0) {
    seterr("gpt_layer_backward: bad layer %d", l);
    return -1;
  }
  return c->bf16 ? layer_bwd_impl<bf16>(c, l, P, G) : layer_bwd_impl<float>(c, l, P, G);
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
