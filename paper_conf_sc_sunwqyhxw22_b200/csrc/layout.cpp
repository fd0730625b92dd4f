// Size table and packed per-layer layout ("for each DNN layer,
// STRONGHOLD also computes the required storage size for the parameter tensors and the
// associated gradients and optimizer states").
#include <cstdarg>
#include <cstdio>
#include <cstring>

#include "sh_internal.hpp"

namespace sh {

static thread_local std::string g_last_error;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
}
void clear_error() { g_last_error.clear(); }
const char* last_error_cstr() { return g_last_error.c_str(); }

bool make_layout(const sh_layer_shape& s, LayerLayout* out) {
  if (s.n_tensors < 1 || s.n_tensors > 64 || s.numel == nullptr) {
    set_error("layer shape: n_tensors must be in 1..64 with a numel array (got %d)", s.n_tensors);
    return false;
  }
  LayerLayout L;
  L.n_tensors = s.n_tensors;
  L.numel.assign(s.numel, s.numel + s.n_tensors);
  L.wd.resize(s.n_tensors);
  for (int k = 0; k < s.n_tensors; ++k) {
    if (L.numel[k] <= 0) {
      set_error("layer shape: tensor %d has numel %lld <= 0", k, (long long)L.numel[k]);
      return false;
    }
    L.wd[k] = s.weight_decay ? (s.weight_decay[k] != 0) : 0;
    L.n_raw += L.numel[k];
  }
  L.offset.assign(s.n_tensors, 0);
  int64_t off = 0;
  for (int pass = 0; pass < 2; ++pass) {  // decayed tensors first, caller order within a class
    for (int k = 0; k < s.n_tensors; ++k) {
      if ((pass == 0) != (L.wd[k] != 0)) continue;
      L.offset[k] = off;
      off += (L.numel[k] + kPad - 1) / kPad * kPad;
    }
    if (pass == 0) L.n_decay = off;
  }
  L.n_pad = off;
  *out = std::move(L);
  return true;
}

void pack_layer(const LayerLayout& L, const float* src, float* dst) {
  std::memset(dst, 0, sizeof(float) * L.n_pad);
  int64_t s = 0;
  for (int k = 0; k < L.n_tensors; ++k) {
    if (src) std::memcpy(dst + L.offset[k], src + s, sizeof(float) * L.numel[k]);
    s += L.numel[k];
  }
}

void unpack_layer(const LayerLayout& L, const float* src, float* dst) {
  int64_t s = 0;
  for (int k = 0; k < L.n_tensors; ++k) {
    std::memcpy(dst + s, src + L.offset[k], sizeof(float) * L.numel[k]);
    s += L.numel[k];
  }
}

void unpack_layer_u16(const LayerLayout& L, const uint16_t* src, uint16_t* dst) {
  int64_t s = 0;
  for (int k = 0; k < L.n_tensors; ++k) {
    std::memcpy(dst + s, src + L.offset[k], sizeof(uint16_t) * L.numel[k]);
    s += L.numel[k];
  }
}

}  // namespace sh
