/*
 * sh_gpt.h -- GPT-2 block compute used to DRIVE the offload engine (bench + parity tests).
 *
 * OUTSIDE THE HOT PATH (BASELINE.json north_star: "the transformer-block GEMMs go through
 * cuBLASLt, are outside the hot path and are labelled as such").  This library is the
 * stand-in for the user's unmodified model code: it reads the parameter
 * pointers the engine's hooks return and writes fp32 gradients into the engine's gradient
 * slots.  It computes the model of DESIGN.md reading R1 (GPT-2 pre-LN, tied embedding,
 * learned positions, tanh GELU, mean token cross entropy) with layer-wise activation
 * checkpointing: only each layer's input x_l (fp32) is kept; BP recomputes the
 * layer's forward (PAPER.md:153 fn. 2).
 *
 * Precision: SH_FP32 (fp32 everywhere, CUBLAS_COMPUTE_32F, no TF32) or SH_BF16_MIXED (bf16
 * weights and GEMM activations, fp32 accumulation, fp32 residual stream, LN statistics,
 * softmax, cross entropy and weight gradients).
 *
 * Determinism: every reduction has a fixed order (cuBLAS with a fixed workspace, fixed-tree
 * kernels, no float atomics; the embedding backward sorts token ids stably), so the same
 * parameters and tokens give bit-identical gradients regardless of which ring slot holds the
 * layer -- the precondition of the engine's bit-exact-across-window property.
 *
 * Layer tensor order (10-12 pointers): ln1_g, ln1_b, w_qkv[3h,h], b_qkv, w_o[h,h], b_o,
 * ln2_g, ln2_b, w_fc[4h,h], b_fc, w_proj[h,4h], b_proj.  Resident order: wte[V,h],
 * wpe[s,h], lnf_g, lnf_b.  Parameters are in the compute dtype, gradients fp32.
 * Tokens are device int32 [B, S+1]: inputs [:, :S], targets [:, 1:].
 * All calls are asynchronous on the configured stream; return 0 on success, else a negative
 * code with gpt_last_error() describing it.
 */
#ifndef SH_GPT_H_
#define SH_GPT_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gpt_ctx gpt_ctx;

typedef struct {
  int32_t n_layers, hidden, heads, seq, max_batch, vocab;
  int32_t precision;  /* SH_FP32 = 0, SH_BF16_MIXED = 1 */
  int32_t device;
  void* stream;       /* cudaStream_t: the engine's compute stream */
} gpt_config;

int32_t gpt_create(const gpt_config* cfg, gpt_ctx** out);
int32_t gpt_destroy(gpt_ctx* ctx);
const char* gpt_last_error(void);
/* Number of this library's own kernel launches (cuBLAS / CUB launches not counted). */
int64_t gpt_kernel_launches(void);
/* Device bytes of activations/workspace held by the context. */
int64_t gpt_workspace_bytes(const gpt_ctx* ctx);

/* x_0 = wte[tok] + wpe[pos]; sets the batch size B (<= max_batch) for this step. */
int32_t gpt_embed_forward(gpt_ctx* ctx, const int32_t* d_tokens, int32_t batch, void* const* res_params);
/* x_{l+1} = block_l(x_l) (checkpoint x_l kept). */
int32_t gpt_layer_forward(gpt_ctx* ctx, int32_t layer, void* const* params);
/* loss = mean CE(LN_f(x_L) wte^T, targets) -> *d_loss (device float); writes dL/dx_L into the
 * residual-gradient buffer, res_grads[2..3] (LN_f) and the head part of res_grads[0] (=). */
int32_t gpt_head_forward_backward(gpt_ctx* ctx, const int32_t* d_tokens, void* const* res_params,
                                  float* const* res_grads, float* d_loss);
/* Forward-only head (inference): loss = mean CE(LN_f(x_L) wte^T, targets) -> *d_loss. */
int32_t gpt_head_forward(gpt_ctx* ctx, const int32_t* d_tokens, void* const* res_params, float* d_loss);
/* Recompute block_l forward from x_l, then backward: fp32 weight grads written into grads[],
 * the residual gradient is propagated in place (dL/dx_{l+1} -> dL/dx_l). */
int32_t gpt_layer_backward(gpt_ctx* ctx, int32_t layer, void* const* params, float* const* grads);
/* res_grads[0][tok] += dL/dx_0 rows (stable, deterministic); res_grads[1][pos] += Σ_b rows. */
int32_t gpt_embed_backward(gpt_ctx* ctx, const int32_t* d_tokens, float* const* res_grads);

/* Staged block, for callers that substitute the attention core (e.g. a fused flash-attention
 * library kernel on the bf16 path).  Forward: forward_qkv (LN1 + QKV GEMM -> buffer 0, [N,3h],
 * columns [q|k|v], head j at j*hd) ; caller writes buffer 1 = causal attention output [N,h] ;
 * forward_out(write_out) (W_o + residual, LN2, MLP; write_out = 0 during the backward recompute).
 * Backward (after the recompute): backward_mlp (MLP, LN2, W_o grads; d_att -> buffer 2 [N,h]) ;
 * caller writes buffer 3 = d qkv [N,3h] ; backward_qkv (W_qkv grads, LN1, residual gradient). */
int32_t gpt_layer_forward_qkv(gpt_ctx* ctx, int32_t layer, void* const* params);
int32_t gpt_layer_forward_out(gpt_ctx* ctx, int32_t layer, void* const* params, int32_t write_out);
int32_t gpt_layer_backward_mlp(gpt_ctx* ctx, int32_t layer, void* const* params, float* const* grads);
int32_t gpt_layer_backward_qkv(gpt_ctx* ctx, int32_t layer, void* const* params, float* const* grads);
/* 0: qkv [N,3h], 1: att [N,h], 2: d_att [N,h], 3: d_qkv [N,3h] (compute dtype, device). */
void* gpt_buffer(gpt_ctx* ctx, int32_t which);

/* Device pointer of checkpoint x_l (fp32 [B*S, h]), l in 0..n_layers (diagnostics / tests). */
float* gpt_checkpoint(gpt_ctx* ctx, int32_t l);

#ifdef __cplusplus
}
#endif
#endif /* SH_GPT_H_ */
