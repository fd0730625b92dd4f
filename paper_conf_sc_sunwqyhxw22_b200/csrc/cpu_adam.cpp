// CPU AdamW of the concurrent optimizer pool (§III-E1) and the bf16 shadow
// writer.  Executes exactly the op sequence of K2 (kernels.cu) in IEEE fp32 so that a layer
// updated here is bit-identical to the same layer updated on the GPU (DESIGN.md "Engine
// numerics"; the property behind PAPER.md:87's "no stale updates, no precision change").
//
// Built with -ffp-contract=off and without -ffast-math: no implicit FMA, no reassociation,
// no FTZ/DAZ (MXCSR defaults).  FMAs are explicit (std::fmaf / _mm512_fmadd_ps, both
// correctly rounded).  bf16 rounding is round-to-nearest, ties AWAY from zero (RNA, R25), by
// integer arithmetic on the fp32 pattern: (u + 0x8000) >> 16, canonical NaN 0x7FC0 -- the rounding
// that makes the split master below lossless (vcvtneps2bf16 is RNE and flushes denormals: not used).
//
// Split master (bf16 host layout, R25): a host-optimised layer keeps its fp32 master as two
// 16-bit planes, hi = rna_bf16(p) -- the compute copy itself, which the H2D prefetch moves at 2 B/param
// -- and lo = the low 16 bits of p's pattern.  Under RNA the fp32 patterns rounding to one bf16 value
// hi are exactly [(hi << 16) - 0x8000, (hi << 16) + 0x7fff], so p = (hi << 16) + sext16(lo): lossless
// for every non-NaN p (a NaN comes back as a NaN), with no shadow copy (12 B/param of host RAM, not 14).
#include <immintrin.h>

#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "sh_internal.hpp"

namespace sh {
namespace cpu {

uint16_t rna_bf16(float x) {
  uint32_t u;
  std::memcpy(&u, &x, 4);
  if ((u & 0x7fffffffu) > 0x7f800000u) return 0x7fc0u;
  return (uint16_t)((u + 0x8000u) >> 16);
}

static inline float join_master(uint16_t hi, uint16_t lo) {
  const uint32_t u = ((uint32_t)hi << 16) + (uint32_t)(int32_t)(int16_t)lo;
  float f;
  std::memcpy(&f, &u, 4);
  return f;
}

static inline void split_master(float p, uint16_t* hi, uint16_t* lo) {
  uint32_t u;
  std::memcpy(&u, &p, 4);
  *hi = rna_bf16(p);
  *lo = (uint16_t)(u & 0xffffu);
}

static inline void adam_scalar(float& p, float& m, float& v, float g, const sh_adam_scalars& s,
                               bool wd, bool use_coef, float coef) {
  if (use_coef) g = g * coef;
  m = std::fmaf(s.beta1, m, s.omb1 * g);
  v = std::fmaf(s.beta2, v, s.omb2 * (g * g));
  const float d = std::sqrt(v) / s.sqrt_bc2 + s.eps;
  const float pp = wd ? p * s.decay : p;
  p = std::fmaf(-s.step_size, m / d, pp);
}

static void adam_scalar_range(float* p, float* m, float* v, const float* g, uint16_t* out16,
                              int64_t b, int64_t e, int64_t n_decay, const sh_adam_scalars& s,
                              bool use_coef, float coef) {
  for (int64_t i = b; i < e; ++i) {
    adam_scalar(p[i], m[i], v[i], g[i], s, i < n_decay, use_coef, coef);
    if (out16) out16[i] = rna_bf16(p[i]);
  }
}

__attribute__((target("avx512f"))) static inline __m256i rna_bf16_16(__m512 x) {
  const __m512i u = _mm512_castps_si512(x);
  const __m512i c8000 = _mm512_set1_epi32(0x8000);
  const __m512i absm = _mm512_set1_epi32(0x7fffffff);
  const __m512i inf = _mm512_set1_epi32(0x7f800000);
  const __m512i qnan = _mm512_set1_epi32(0x7fc0);
  __m512i r = _mm512_srli_epi32(_mm512_add_epi32(u, c8000), 16);
  const __mmask16 nan = _mm512_cmpgt_epu32_mask(_mm512_and_si512(u, absm), inf);
  r = _mm512_mask_mov_epi32(r, nan, qnan);
  return _mm512_cvtepi32_epi16(r);
}

// Software-prefetch distance of the AVX-512 AdamW in elements (SH_CPU_PF, default 512; 0: off).  The
// L2 streamer stops at every 4 KiB page boundary, which the kernel's concurrent streams (5 read + 4
// written on the split master) cross every 64-128 iterations; prefetching 512 elements ahead on every
// read stream keeps each core's misses in flight across them.  Measured on the B200 box
// (profiles/r02_cpu_pf.jsonl): the split AdamW alone 143-165 -> 176-180 GB/s at 12 threads, beside
// H2D + D2H DMA 187-192 -> 196-198 GB/s of host-DRAM total; c4max 5.31-5.46 -> 5.61 samples/s.
static int64_t prefetch_distance() {
  static const int64_t d = [] {
    const char* e = getenv("SH_CPU_PF");
    const long long x = e ? atoll(e) : 512;
    return (int64_t)(x > 0 ? (x + 31) / 32 * 32 : 0);
  }();
  return d;
}

template <bool kWd, bool kCoef, bool kOut, bool kNT>
__attribute__((target("avx512f"))) static void adam_avx512_block(
    float* __restrict p, float* __restrict m, float* __restrict v, const float* __restrict g,
    uint16_t* __restrict out16, int64_t b, int64_t e, const sh_adam_scalars& s, float coef) {
  const __m512 b1 = _mm512_set1_ps(s.beta1), b2 = _mm512_set1_ps(s.beta2);
  const __m512 omb1 = _mm512_set1_ps(s.omb1), omb2 = _mm512_set1_ps(s.omb2);
  const __m512 eps = _mm512_set1_ps(s.eps), nss = _mm512_set1_ps(-s.step_size);
  const __m512 sbc2 = _mm512_set1_ps(s.sqrt_bc2), decay = _mm512_set1_ps(s.decay);
  const __m512 vc = _mm512_set1_ps(coef);
  const int64_t pf = prefetch_distance();
  for (int64_t i = b; i < e; i += 16) {
    if (pf > 0 && i + pf < e) {
      _mm_prefetch(reinterpret_cast<const char*>(g + i + pf), _MM_HINT_T0);
      _mm_prefetch(reinterpret_cast<const char*>(m + i + pf), _MM_HINT_T0);
      _mm_prefetch(reinterpret_cast<const char*>(v + i + pf), _MM_HINT_T0);
      _mm_prefetch(reinterpret_cast<const char*>(p + i + pf), _MM_HINT_T0);
    }
    __m512 gg = _mm512_loadu_ps(g + i);
    if (kCoef) gg = _mm512_mul_ps(gg, vc);
    __m512 mm = _mm512_loadu_ps(m + i);
    __m512 vv = _mm512_loadu_ps(v + i);
    __m512 pp = _mm512_loadu_ps(p + i);
    mm = _mm512_fmadd_ps(b1, mm, _mm512_mul_ps(omb1, gg));
    vv = _mm512_fmadd_ps(b2, vv, _mm512_mul_ps(omb2, _mm512_mul_ps(gg, gg)));
    const __m512 d = _mm512_add_ps(_mm512_div_ps(_mm512_sqrt_ps(vv), sbc2), eps);
    if (kWd) pp = _mm512_mul_ps(pp, decay);
    pp = _mm512_fmadd_ps(nss, _mm512_div_ps(mm, d), pp);
    _mm512_storeu_ps(m + i, mm);
    _mm512_storeu_ps(v + i, vv);
    _mm512_storeu_ps(p + i, pp);
    if (kOut) {
      // the shadow is written once and next read by the H2D DMA: stream it (no read-for-ownership)
      if (kNT) _mm256_stream_si256(reinterpret_cast<__m256i*>(out16 + i), rna_bf16_16(pp));
      else _mm256_storeu_si256(reinterpret_cast<__m256i*>(out16 + i), rna_bf16_16(pp));
    }
  }
}

template <bool kWd>
static void adam_vec_dispatch(float* p, float* m, float* v, const float* g, uint16_t* out16,
                              int64_t b, int64_t e, const sh_adam_scalars& s, bool use_coef,
                              float coef) {
  const bool nt = out16 && ((reinterpret_cast<uintptr_t>(out16 + b) & 31) == 0);
  if (use_coef) {
    if (!out16) adam_avx512_block<kWd, true, false, false>(p, m, v, g, out16, b, e, s, coef);
    else if (nt) adam_avx512_block<kWd, true, true, true>(p, m, v, g, out16, b, e, s, coef);
    else adam_avx512_block<kWd, true, true, false>(p, m, v, g, out16, b, e, s, coef);
  } else {
    if (!out16) adam_avx512_block<kWd, false, false, false>(p, m, v, g, out16, b, e, s, coef);
    else if (nt) adam_avx512_block<kWd, false, true, true>(p, m, v, g, out16, b, e, s, coef);
    else adam_avx512_block<kWd, false, true, false>(p, m, v, g, out16, b, e, s, coef);
  }
}

bool has_avx512() {
  static const bool ok = __builtin_cpu_supports("avx512f");
  return ok;
}

void adamw_range(float* p, float* m, float* v, const float* g, uint16_t* out16, int64_t begin,
                 int64_t end, int64_t n_decay, const sh_adam_scalars& sc, bool use_coef,
                 float coef) {
  if (!has_avx512()) {
    adam_scalar_range(p, m, v, g, out16, begin, end, n_decay, sc, use_coef, coef);
    return;
  }
  // decayed part [begin, min(end, n_decay)), then the rest; vector body in 16s, scalar tails
  const int64_t split = end < n_decay ? end : (begin > n_decay ? begin : n_decay);
  const int64_t parts[2][2] = {{begin, split}, {split, end}};
  for (int k = 0; k < 2; ++k) {
    const int64_t b = parts[k][0], e = parts[k][1];
    if (b >= e) continue;
    const int64_t ev = b + ((e - b) / 16) * 16;
    if (k == 0) adam_vec_dispatch<true>(p, m, v, g, out16, b, ev, sc, use_coef, coef);
    else adam_vec_dispatch<false>(p, m, v, g, out16, b, ev, sc, use_coef, coef);
    adam_scalar_range(p, m, v, g, out16, ev, e, n_decay, sc, use_coef, coef);
  }
  if (out16) _mm_sfence();  // order the streamed shadow before the caller's release of ready[j]
}

__attribute__((target("avx512f"))) static void cast_avx512(const float* src, uint16_t* dst,
                                                           int64_t b, int64_t e) {
  for (int64_t i = b; i < e; i += 16)
    _mm256_storeu_si256(reinterpret_cast<__m256i*>(dst + i), rna_bf16_16(_mm512_loadu_ps(src + i)));
}

void cast_bf16_range(const float* src, uint16_t* dst, int64_t begin, int64_t end) {
  int64_t ev = begin;
  if (has_avx512()) {
    ev = begin + ((end - begin) / 16) * 16;
    cast_avx512(src, dst, begin, ev);
  }
  for (int64_t i = ev; i < end; ++i) dst[i] = rna_bf16(src[i]);
}

// ---- split master -----------------------------------------------------------------------------
static void adam_split_scalar_range(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t b,
                                    int64_t e, int64_t n_decay, const sh_adam_scalars& s, bool use_coef,
                                    float coef) {
  for (int64_t i = b; i < e; ++i) {
    float p = join_master(hi[i], lo[i]);
    adam_scalar(p, m[i], v[i], g[i], s, i < n_decay, use_coef, coef);
    split_master(p, hi + i, lo + i);
  }
}

template <bool kWd, bool kCoef>
__attribute__((target("avx512f,avx512bw"))) static void adam_split_avx512_block(
    uint16_t* __restrict hi, uint16_t* __restrict lo, float* __restrict m, float* __restrict v,
    const float* __restrict g, int64_t b, int64_t e, const sh_adam_scalars& s, float coef) {
  const __m512 b1 = _mm512_set1_ps(s.beta1), b2 = _mm512_set1_ps(s.beta2);
  const __m512 omb1 = _mm512_set1_ps(s.omb1), omb2 = _mm512_set1_ps(s.omb2);
  const __m512 eps = _mm512_set1_ps(s.eps), nss = _mm512_set1_ps(-s.step_size);
  const __m512 sbc2 = _mm512_set1_ps(s.sqrt_bc2), decay = _mm512_set1_ps(s.decay);
  const __m512 vc = _mm512_set1_ps(coef);
  const int64_t pf = prefetch_distance();
  for (int64_t i = b; i < e; i += 16) {
    if (pf > 0 && i + pf < e) {  // the five read streams (hi / lo: one line per 32 elements)
      _mm_prefetch(reinterpret_cast<const char*>(g + i + pf), _MM_HINT_T0);
      _mm_prefetch(reinterpret_cast<const char*>(m + i + pf), _MM_HINT_T0);
      _mm_prefetch(reinterpret_cast<const char*>(v + i + pf), _MM_HINT_T0);
      if ((i & 31) == 0) {
        _mm_prefetch(reinterpret_cast<const char*>(hi + i + pf), _MM_HINT_T0);
        _mm_prefetch(reinterpret_cast<const char*>(lo + i + pf), _MM_HINT_T0);
      }
    }
    const __m512i h = _mm512_cvtepu16_epi32(_mm256_loadu_si256(reinterpret_cast<const __m256i*>(hi + i)));
    const __m512i l = _mm512_cvtepi16_epi32(_mm256_loadu_si256(reinterpret_cast<const __m256i*>(lo + i)));
    __m512 pp = _mm512_castsi512_ps(_mm512_add_epi32(_mm512_slli_epi32(h, 16), l));
    __m512 gg = _mm512_loadu_ps(g + i);
    if (kCoef) gg = _mm512_mul_ps(gg, vc);
    __m512 mm = _mm512_loadu_ps(m + i);
    __m512 vv = _mm512_loadu_ps(v + i);
    mm = _mm512_fmadd_ps(b1, mm, _mm512_mul_ps(omb1, gg));
    vv = _mm512_fmadd_ps(b2, vv, _mm512_mul_ps(omb2, _mm512_mul_ps(gg, gg)));
    const __m512 d = _mm512_add_ps(_mm512_div_ps(_mm512_sqrt_ps(vv), sbc2), eps);
    if (kWd) pp = _mm512_mul_ps(pp, decay);
    pp = _mm512_fmadd_ps(nss, _mm512_div_ps(mm, d), pp);
    _mm512_storeu_ps(m + i, mm);
    _mm512_storeu_ps(v + i, vv);
    _mm256_storeu_si256(reinterpret_cast<__m256i*>(hi + i), rna_bf16_16(pp));
    _mm256_storeu_si256(reinterpret_cast<__m256i*>(lo + i), _mm512_cvtepi32_epi16(_mm512_castps_si512(pp)));
  }
}

void adamw_range_split(uint16_t* hi, uint16_t* lo, float* m, float* v, const float* g, int64_t begin, int64_t end,
                       int64_t n_decay, const sh_adam_scalars& sc, bool use_coef, float coef) {
  if (!has_avx512()) {
    adam_split_scalar_range(hi, lo, m, v, g, begin, end, n_decay, sc, use_coef, coef);
    return;
  }
  const int64_t split = end < n_decay ? end : (begin > n_decay ? begin : n_decay);
  const int64_t parts[2][2] = {{begin, split}, {split, end}};
  for (int k = 0; k < 2; ++k) {
    const int64_t b = parts[k][0], e = parts[k][1];
    if (b >= e) continue;
    const int64_t ev = b + ((e - b) / 16) * 16;
    if (k == 0) {
      if (use_coef) adam_split_avx512_block<true, true>(hi, lo, m, v, g, b, ev, sc, coef);
      else adam_split_avx512_block<true, false>(hi, lo, m, v, g, b, ev, sc, coef);
    } else {
      if (use_coef) adam_split_avx512_block<false, true>(hi, lo, m, v, g, b, ev, sc, coef);
      else adam_split_avx512_block<false, false>(hi, lo, m, v, g, b, ev, sc, coef);
    }
    adam_split_scalar_range(hi, lo, m, v, g, ev, e, n_decay, sc, use_coef, coef);
  }
}

void split_range(const float* src, uint16_t* hi, uint16_t* lo, int64_t begin, int64_t end) {
  for (int64_t i = begin; i < end; ++i) split_master(src[i], hi + i, lo + i);
}

void join_range(const uint16_t* hi, const uint16_t* lo, float* dst, int64_t begin, int64_t end) {
  for (int64_t i = begin; i < end; ++i) dst[i] = join_master(hi[i], lo[i]);
}

}  // namespace cpu
}  // namespace sh
