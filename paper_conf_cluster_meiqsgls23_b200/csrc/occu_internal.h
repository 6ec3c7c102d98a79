// Internal declarations shared by the runtime (occu_runtime.cu), the host
// packer (pack.cpp), the weights code (weights.cpp) and the kernels.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/occu.h"

struct ncclComm;

namespace occu {

// Thread-local error for calls that have no ctx (occu_pack, occu_nccl_unique_id).
void set_global_error(const std::string &msg);
const char *global_error();

// Set-Transformer decoder parameters (readout = OCCU_READOUT_SET_DECODER), offsets in floats
// into the flat parameter vector (file order, occu_gen/weights.py).
struct FfnOff { size_t W1, b1, W2, b2; };
struct MabOff { size_t Wq, bq, Wk, bk, Wv, bv, Wo, bo, ln1_g, ln1_b; FfnOff F; size_t ln2_g, ln2_b; };
struct DecLayout { size_t S; FfnOff P; MabOff M1, M2; FfnOff D; };
// Graphormer layer (NEXT-3): ln1, MHA (Wq bq Wk bk Wv bv Wo bo), ln2, FFN.
struct GphOff { size_t ln1_g, ln1_b, Wq, bq, Wk, bk, Wv, bv, Wo, bo, ln2_g, ln2_b; FfnOff F; };

struct ParamLayout {
  // offsets (in floats) of each tensor inside the flat parameter vector
  std::vector<size_t> W_u, W_e, W_m, a_s, a_d;
  size_t W_1 = 0, b_1 = 0, w_2 = 0, b_2 = 0, total = 0;
  std::vector<int> d_in, de_in;
  bool dec = false;
  DecLayout D{};
  std::vector<GphOff> G;    // Graphormer layers
  int head_in = 0;          // W_1 columns: d (mean readout) or k·d (decoder)
};
ParamLayout make_layout(const occu_config &c);

// Grow-only device buffer.
struct DevBuf {
  void *ptr = nullptr;
  size_t bytes = 0;
  cudaError_t ensure(size_t need);
  void release();
  template <class T> T *as() const { return reinterpret_cast<T *>(ptr); }
};

// Device-resident per-layer activations and scratch for one batch size.
struct Workspace {
  // inputs staged on device (host-pointer calls)
  DevBuf node_feat, edge_feat, targets, out_occ;
  DevBuf csr;              // concatenated int32 CSR arrays for host-CSR calls
  DevBuf e0;               // edge features permuted to in-CSR order [E][F_e]
  std::vector<DevBuf> hbar, p, q, e, h;   // per layer
  std::vector<DevBuf> gs;                 // per layer channel-softmax gates, kept for the backward (training)
  DevBuf g;                // [E][d] channel-softmax gates (scratch)
  DevBuf rpart;            // [N][d] readout chunk partials (rows written sparsely) when h_L is kept
  DevBuf r, c, yhat;       // [B][d], [B][d_h], [B]
  // backward scratch
  DevBuf dy, dc, dr, dh, dhprev, dP, MG, DV, DZ, deA, deB, dalpha, dpq, partial, loss;
  DevBuf rowexp;           // d = 256: per-row power-of-two scale exponents of node-transform inputs
  DevBuf tcpart;           // tensor-core aggregation: boundary-segment partials
  DevBuf dpart;            // per-warp [da_s; da_d] partials
  DevBuf anf[2], aef[2], acsr[2];   // occu_predict_async / occu_train_step_async: double-buffered input staging
  DevBuf aty[2];           // occu_train_step_async: staged targets
  DevBuf dT, dZ;           // decoder readout: per-node FFN hidden / output rows [N][d]
  DevBuf dprep;            // decoder readout: folded key map M [d][16] and offsets c [16]
  DevBuf dpool;            // decoder readout: pool partials [B][8][16·d + 32]
  std::vector<DevBuf> gh;  // Graphormer layer outputs [N][d] (per layer)
  DevBuf scsr, snf, sef, sdesc;   // occu_synthesize: batch CSR, node / edge rows, descriptors
  DevBuf hf;               // OCCU_BF16 with Graphormer / decoder: h_L widened to FP32 (R41)
  DevBuf gx, gqkv, go;     // Graphormer scratch: LN output [N][d], Q|K|V [3][N][d], attention [N][d]
  std::vector<DevBuf> gsave;   // training: 8 saved [N][d] intermediates per Graphormer layer
  DevBuf gscr;             // training: Graphormer backward scratch 5 x [N][d] + stats
  DevBuf gdh[2];           // training: gradients w.r.t. the stack's node states (ping-pong)
  DevBuf dbwd;             // training: decoder backward rows / stats / partials
  DevBuf hub;              // aggregation: per-64-edge-unit partials of hub segments
  DevBuf rexp;             // backward: row scale exponents of DV [E], DZ [E], dP [N] (producer -> row-GEMM)
  std::vector<DevBuf> hbits;   // training: per layer sign bitmask of h [N][d/32] (LReLU' masks)
  void release_all();
};

struct DevCsr {            // device view of a packed batch
  int32_t B = 0, N = 0, E = 0;
  int32_t max_deg = -1;    // max in-degree (-1 unknown): > HUB_DEG selects the aggregation's hub path
  const int32_t *node_off = nullptr, *edge_off = nullptr, *in_ptr = nullptr, *in_src = nullptr,
                *in_dst = nullptr, *in_eid = nullptr, *out_ptr = nullptr, *out_pos = nullptr,
                *node_graph = nullptr;
};

// Per-kernel CUDA-event profiler (bench.py's roofline numbers).
struct Profiler {
  bool on = false;
  struct Rec { int kind; cudaEvent_t a, b; };
  std::vector<std::string> names;
  std::vector<double> total_ms;
  std::vector<int64_t> count;
  std::vector<Rec> pending;
  std::vector<cudaEvent_t> pool;
  int cur = -1;
  cudaEvent_t cur_a = nullptr;
  cudaStream_t cur_s = nullptr;
  void begin(const char *name, cudaStream_t s);
  void end();
  void drain();          // synchronises and folds pending pairs into totals
  void reset();
  ~Profiler();
};

}  // namespace occu

struct occu_ctx {
  occu_config cfg{};
  occu::ParamLayout layout;
  int device = 0;
  cudaStream_t stream = nullptr;
  int num_sms = 148;
  bool weights_ready = false;
  bool keep = false;
  int path = 0;            // 0: tensor cores, 1: CUDA-core SIMT FP32, 2: tensor cores + fused aggregation
  int l2_order = 1;        // alternate row-walk direction between producer/consumer kernels (L2 reuse)
  // programmatic dependent launch, per kernel family (bit mask, OCCU_PDL): 1 FP32 row-GEMMs,
  // 2 FP32 gather, 4 layer-1 edge, 8 readout, 16 BF16 row-GEMMs, 32 weight images, 64 BF16
  // gather.  Default from A/B runs on CFG2: the FP32 gather and the readout lose with it.
  int pdl = 1 | 4 | 16 | 32 | 64;
  int fuse_edge_gate = 0;  // path 0: edge transform + gate in one kernel (edgegate_kernel), OCCU_FUSE_EG=1
  int fuse_agg = 0;        // path 0 inference: edge transform + gate + message + segmented sum in one
                           // kernel (edgegate_kernel<AGG>; g never reaches HBM), OCCU_FUSE_EGA
  occu::DevBuf wimg, wjobs, wfexp;   // prebuilt tensor-core weight images (per parameter version)
  int64_t params_version = 0, wimg_version = -1;
  int64_t dprep_version = -1;   // decoder: params version the folded key map was built for
  float weight_decay = 1e-4f;
  occu::DevBuf params, grads, adam_m, adam_v;
  int64_t adam_t = 0;
  occu::Workspace ws;
  occu::DevCsr last_csr;   // geometry of the last forward (for occu_get_tensor)
  bool have_forward = false;
  bool h_last_stored = true;   // false: the last forward kept only readout partials of h_L
  bool small_fwd = false;      // the last forward ran the single-CTA small-batch kernel
  int hbits_layers = 0;        // the last forward wrote the sign bits of h^0 .. h^{hbits_layers-1}
  bool small_enabled = true;   // occu_set_small_batch_kernel: single-CTA forward for tiny batches (default on)
  int64_t launches = 0;
  mutable occu::Profiler prof;
  // occu_predict_async: H2D on a copy stream into staging slot a_slot, compute on `stream`
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t a_copied[2] = {nullptr, nullptr}, a_free[2] = {nullptr, nullptr};
  int a_slot = 0;
  // data parallel
  ncclComm *comm = nullptr;
  int rank = 0, world = 1;
  double nccl_timeout_s = 600.0;   // occu_dist_set_timeout: watchdog on NCCL progress (0 = none)
  bool comm_aborted = false;       // set when the watchdog (or occu_dist_abort) aborted comm
  std::string err;
};

namespace occu {

// ---- programmatic dependent launch (PDL) -------------------------------------
// Kernels launched with launch_pdl may start (prologue: barriers, TMEM, tensor-map
// prefetch) while their predecessor drains; every such kernel calls pdl_trigger()
// first and pdl_wait() before its first global-memory access, so it observes all of
// the predecessor's writes (and, transitively, everything earlier on the stream).
#ifdef __CUDACC__
// The fp16x2 row scale of the tensor-core converters: e such that max|x|·2^e lies in
// [2^14, 2^15), 0 for an all-zero row, capped at 100 (kernels_tc.cu).  Shared so
// that a producer kernel can hand the exponents of its output rows to the next row-GEMM.
__device__ __forceinline__ int occu_row_scale_exp(float mx) {
  if (!(mx > 0.f) || !isfinite(mx)) return 0;
  int E;
  frexpf(mx, &E);
  return min(15 - E, 100);
}
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
template <class... KArgs, class... Args>
cudaError_t launch_pdl(bool pdl, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                       cudaStream_t st, Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}
#endif

#define OCCU_PROF_BEGIN(ctx, name, st) \
  do { if ((ctx)->prof.on) (ctx)->prof.begin(name, st); } while (0)
#define OCCU_PROF_END(ctx) \
  do { if ((ctx)->prof.on) (ctx)->prof.end(); } while (0)

// ---- kernel launchers (kernels_simt.cu) ------------------------------------
struct FwdLayerArgs {
  const float *h_in; int K;            // [N][K]
  const float *e_in; int Ke;           // [E][Ke] in-CSR order
  const float *W_u, *W_e, *W_m, *a_s, *a_d;
  float *hbar, *p, *q, *e_out, *g, *h_out;   // e_out may be null
  // Fused variants (tensor-core path): layer 1 reads edge_feat rows through in_eid
  // (e_eid != null; e0_out, if set, receives the permuted copy for the backward), and
  // the last layer's aggregation emits readout chunk partials into rpart (h_out may
  // then be null).  See gather_segsum_kernel / readout_head_kernel.
  const int32_t *e_eid; float *e0_out; float *rpart;
  bool save_w = false;                 // reading B, training: g receives the softmax weights
  uint32_t *h_bits = nullptr;          // training: sign bitmask of h_out for the backward's LReLU'
  bool infer = false;                  // inference (nothing saved): the fused edge-gate-aggregate kernel may run
};
int launch_forward_layer(const occu_ctx *ctx, const DevCsr &csr, const FwdLayerArgs &a,
                         cudaStream_t st);
bool tc_supported(const occu_config &c);
// Weight images for the tensor-core row-GEMMs; kind: 0 W_u, 1 W_e, 2 W_m, 3 W_mᵀ, 4 W_eᵀ, 5 W_uᵀ.
int tc_prepare_weights(occu_ctx *ctx, cudaStream_t st);
const uint8_t *tc_wimg(const occu_ctx *ctx, int kind, int layer);
const int *tc_wfexp(const occu_ctx *ctx, int kind, int layer);
bool wgrad_tc_supported(int A, int Bn);
int launch_bwd_gate_tc(const occu_ctx *ctx, const DevCsr &csr, int layer, const float *e,
                       const float *dh, const float *h, const float *hbar, float *MG, float *DV,
                       cudaStream_t st);
int launch_plain_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                    const float *add, float *out, const char *name, cudaStream_t st,
                    const float *mask_h = nullptr, const int32_t *in_ptr = nullptr,
                    bool mask_bf = false, const uint32_t *mask_bits = nullptr,
                    const int *rexp = nullptr);
// OCCU_BF16 training: z = W_e e_in recomputed from BF16 e_in on the BF16 tensor-core path
// (as the forward), epilogue dy = de ⊙ e' ⊙ σ(-αz) with BF16 e', dα = <dy, z>, DZ = α dy.
int launch_bwd_edge_bf16(const occu_ctx *ctx, const DevCsr &csr, int layer, const void *e_in,
                         int Ke, const void *e, const float *de, const float *p, const float *q,
                         float *DZ, float *dal, cudaStream_t st);
int launch_bwd_edge_tc(const occu_ctx *ctx, const DevCsr &csr, int layer, const float *e_in, int Ke,
                       const float *e, const float *de, const float *p,
                       const float *q, float *DZ, float *dal, cudaStream_t st,
                       int *dz_rexp = nullptr);
int launch_wgrad_tc(const occu_ctx *ctx, const float *X, int A, const void *Y, int Bn, long R,
                    int splits, float *partial, cudaStream_t st, bool ybf = false);
size_t tc_partial_floats(int E, int D);
int launch_forward_layer_tc(const occu_ctx *ctx, const DevCsr &csr, int layer, const FwdLayerArgs &a,
                            float *partial, cudaStream_t st);
int launch_gather_segsum(const occu_ctx *ctx, const DevCsr &csr, const float *g,
                         const float *hbar, float *h_out, float *rpart, cudaStream_t st,
                         uint32_t *h_bits = nullptr);
// Reading B (OCCU_MSG_NEIGHBOR_SOFTMAX, NEXT-1): v holds the logits W_m e'; the per-channel
// softmax over each destination's in-edges, the message product and the segmented sum in one
// pass; write_w (training) overwrites v with the softmax weights for the backward.
int launch_gather_segsoftmax(const occu_ctx *ctx, const DevCsr &csr, float *v, const float *hbar,
                             float *h_out, float *rpart, bool write_w, cudaStream_t st);
// OCCU_BF16: g, h̄, h stored as BF16 (FP32 arithmetic); rpart stays FP32.
int launch_gather_segsoftmax_bf16(const occu_ctx *ctx, const DevCsr &csr, void *v, const void *hbar,
                                  void *h_out, float *rpart, bool write_w, cudaStream_t st);
int launch_gather_segsum_bf16(const occu_ctx *ctx, const DevCsr &csr, const void *g,
                              const void *hbar, void *h_out, float *rpart, cudaStream_t st,
                              uint32_t *h_bits = nullptr);
// OCCU_BF16 forward layer (kernels_bf16.cu); FwdLayerArgs pointers to h̄, e', g, h hold BF16.
int launch_pair_bf16(const occu_ctx *ctx, int epi, bool af32, const void *A, int K, int R, int layer,
                     void *out, const float *a_s, const float *a_d, float *p, float *q,
                     const int32_t *src, const int32_t *dst, const char *name, cudaStream_t st);
int launch_forward_layer_bf16(const occu_ctx *ctx, const DevCsr &csr, int layer,
                              const FwdLayerArgs &a, cudaStream_t st);
int launch_permute_rows(const occu_ctx *ctx, const float *src, const int32_t *idx, int rows,
                        int width, float *dst, cudaStream_t st);
// h: [N][d] last-layer states, or (chunked) the readout chunk partials of
// gather_segsum_kernel (row min(u1 - 1, 8c + 7) holds graph b's sum over chunk c).
int launch_readout_head(const occu_ctx *ctx, const DevCsr &csr, const float *h, bool chunked,
                        const float *params, float *r, float *c, float *yhat, cudaStream_t st);
// NEXT-2 readout (kernels_decoder.cu): Z = FFN(h_L) on tensor cores (T = ReLU(h W1ᵀ + b1),
// Z = T W2ᵀ + b2), then per graph the k-seed attention pool over Z, the MAB / SAB / FFN tail
// and the head; r receives the flattened decoder output [B][k·d].
int launch_bf16_to_f32(const occu_ctx *ctx, const void *src, size_t n, float *dst, cudaStream_t st);
bool small_forward_ok(const occu_ctx *ctx, const DevCsr &csr);
int launch_small_forward(const occu_ctx *ctx, const DevCsr &csr, const float *nf, const float *ef,
                         float *r, float *cvec, float *yhat, cudaStream_t st);
// Graphormer layer intermediates kept for the backward (training): LN1 output, Q, K, V, the
// attention output (before W_o), h̄, LN2 output, FFN hidden (post-ReLU), all [N][d].
struct GphSave { float *X1, *Q, *K, *V, *O, *Hb, *X2, *T; };
int launch_graphormer_layer(const occu_ctx *ctx, const DevCsr &csr, int j, const float *h_in,
                            float *h_out, float *X, float *QKV, float *O, cudaStream_t st,
                            const GphSave *sv = nullptr);
// Backward of Graphormer layer j (kernels_stack.cu): dout = ∂L/∂(layer output) -> dh_in
// (∂L/∂h_in), parameter gradients into ctx->grads.  scratch: 5 x [N][d].
int launch_graphormer_layer_bwd(occu_ctx *ctx, const DevCsr &csr, int j, const float *h_in,
                                const GphSave &sv, const float *dout, float *dh_in, float *scratch,
                                cudaStream_t st);
// dA = dh ⊙ LReLU'(h) (÷ deg for MEAN), the last ANEE layer's aggregation gradient from the
// gradient of its output h (kernels_stack.cu).
int launch_mask_dA(const occu_ctx *ctx, const DevCsr &csr, const float *dh, const float *h, float *dA,
                   cudaStream_t st);
// Row-GEMM out = (A Wᵀ [+ add]) ⊙ (mask > 0 ? 1 : slope) with a prebuilt image (no ÷deg).
int launch_plain_masked_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                           const float *add, float *out, const char *name, cudaStream_t st,
                           const float *mask, float slope);
// NEXT-2 training (kernels_decoder.cu): backward of the decoder readout from dr = ∂L/∂r
// [B][k·d] down to dhL = ∂L/∂(the decoder's node-state input hL) [N][d]; T, Z: the forward's
// FFN hidden / output rows; dZ, dT: [N][d] scratch.  Parameter gradients into ctx->grads.
int launch_set_decoder_bwd(occu_ctx *ctx, const DevCsr &csr, const float *hL, const float *T,
                           const float *Z, const float *dr, float *dZ, float *dT, float *dhL,
                           cudaStream_t st);
// out[c] = Σ_r X[r][c] over R rows of width d, fixed order (kernels_stack.cu)
int launch_colsum_rows(occu_ctx *ctx, const float *X, long R, float *out, cudaStream_t st);
// LayerNorm parameter gradients over R rows (x = LN input, gamma its gain): dγ = Σ dy ⊙ x̂,
// dβ = Σ dy (fixed order); dx_scratch [R][d] receives the (unused) input gradient.
int launch_ln_param_grads(occu_ctx *ctx, const float *x, const float *gam, const float *dy, long R,
                          float *dx_scratch, float *gg, float *gb, cudaStream_t st);
// Image slot of Graphormer layer j's transposed matrices (kinds 0-5: W_qᵀ W_kᵀ W_vᵀ W_oᵀ W1ᵀ W2ᵀ).
int gph_tslot(const occu_config &c, int j);
int launch_bias_add_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                       const float *bias, const float *add, float *out, const char *name,
                       cudaStream_t st);
int launch_set_decoder(const occu_ctx *ctx, const DevCsr &csr, const float *hL, float *T, float *Z,
                       float *r, float *c, float *yhat, cudaStream_t st);
// Row-GEMM out = act(A Wᵀ + bias) over R rows on tensor cores with a prebuilt image (kernels_tc.cu).
int launch_bias_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                   const float *bias, bool relu, float *out, const char *name, cudaStream_t st);

struct BwdLayerArgs {
  int layer;
  const float *h_in; int K;           // h^{i-1} [N][K]
  const float *e_in; int Ke;          // e^{i-1} [E][Ke]
  const float *hbar, *p, *q, *e, *h;  // layer i saved
  const float *g;                     // layer i gates saved by the forward (nullable: recompute)
  const float *dh;                    // [N][d] gradient w.r.t. h^i
  const float *de_out;                // [E][d] gradient w.r.t. e^i from layer i+1 (nullable)
  float *de_prev;                     // [E][Ke] (nullable at layer 0)
  float *dh_prev;                     // [N][K]  (nullable at layer 0)
  const uint32_t *h_in_bits = nullptr;  // sign bitmask of h_in (gather_segsum, training forward):
                                      // LReLU'(h^{i-1}) for dh_prev without re-reading h_in rows
  bool bf = false;                    // OCCU_BF16: hbar, e, g, h and (layer > 0) h_in, e_in
                                      // point to BF16 rows; gradients stay FP32 (R28)
};
int launch_backward_layer(occu_ctx *ctx, const DevCsr &csr, const BwdLayerArgs &a,
                          cudaStream_t st);
// the backward's weight-gradient dispatcher (kernels_simt.cu), exported for occu_test_wgrad
int launch_wgrad(occu_ctx *ctx, const float *X, int A, const void *Y, int Bn, long R, float *out,
                 cudaStream_t st, bool ybf);
int launch_head_backward(occu_ctx *ctx, const DevCsr &csr, const float *targets, int global_B,
                         cudaStream_t st);
int launch_adam(occu_ctx *ctx, float lr, cudaStream_t st);

}  // namespace occu
