// C-ABI runtime: context, weights, device batches, forward / train-step
// orchestration, NCCL data parallelism and introspection (include/occu.h).
#include <cuda_runtime.h>
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sched.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <string>
#include <vector>

#include "nccl.h"
#include "occu_internal.h"

void occu_host_batch_release(occu_csr_batch *b);

namespace occu {
void init_flat(const occu_config &c, uint64_t seed, std::vector<float> &out);
bool write_file(const char *path, const char magic[8], const occu_config &c,
                const std::vector<std::pair<const void *, size_t>> &chunks, std::string &err);
occu_status read_file(const char *path, const char magic[8], const occu_config &c,
                      std::vector<unsigned char> &payload, size_t expect_bytes, std::string &err);

static thread_local std::string g_err;
void set_global_error(const std::string &msg) { g_err = msg; }
const char *global_error() { return g_err.c_str(); }

cudaError_t DevBuf::ensure(size_t need) {
  if (need == 0) need = 16;
  if (bytes >= need) return cudaSuccess;
  if (ptr) cudaFree(ptr);
  ptr = nullptr;
  bytes = 0;
  const size_t cap = need + need / 8;
  cudaError_t e = cudaMalloc(&ptr, cap);
  if (e == cudaSuccess) bytes = cap;
  else ptr = nullptr;
  return e;
}
void DevBuf::release() {
  if (ptr) cudaFree(ptr);
  ptr = nullptr;
  bytes = 0;
}
void Workspace::release_all() {
  DevBuf *bufs[] = {&node_feat, &edge_feat, &targets, &out_occ, &csr, &e0, &g, &r, &c, &yhat,
                    &dy, &dc, &dr, &dh, &dhprev, &dP, &MG, &DV, &DZ, &deA, &deB, &dalpha,
                    &dpq, &partial, &loss, &tcpart, &dpart, &rpart, &anf[0], &anf[1],
                    &aef[0], &aef[1], &acsr[0], &acsr[1], &dT, &dZ, &dprep, &dpool, &gx, &gqkv, &go, &gscr, &gdh[0], &gdh[1], &dbwd, &hub, &aty[0], &aty[1], &rowexp,
                    &scsr, &snf, &sef, &sdesc, &hf};
  for (DevBuf *b : bufs) b->release();
  for (auto *v : {&hbar, &p, &q, &e, &h, &gs, &gh, &gsave, &hbits})
    for (DevBuf &b : *v) b.release();
}

void Profiler::begin(const char *name, cudaStream_t s) {
  int k = -1;
  for (size_t i = 0; i < names.size(); ++i)
    if (names[i] == name) { k = int(i); break; }
  if (k < 0) {
    names.push_back(name);
    total_ms.push_back(0.0);
    count.push_back(0);
    k = int(names.size()) - 1;
  }
  cudaEvent_t a;
  if (!pool.empty()) { a = pool.back(); pool.pop_back(); }
  else cudaEventCreate(&a);
  cudaEventRecord(a, s);
  cur = k;
  cur_a = a;
  cur_s = s;
}
void Profiler::end() {
  if (cur < 0) return;
  cudaEvent_t b;
  if (!pool.empty()) { b = pool.back(); pool.pop_back(); }
  else cudaEventCreate(&b);
  cudaEventRecord(b, cur_s);
  pending.push_back({cur, cur_a, b});
  cur = -1;
  if (pending.size() > 4096) drain();
}
void Profiler::drain() {
  for (Rec &r : pending) {
    cudaEventSynchronize(r.b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, r.a, r.b);
    total_ms[r.kind] += ms;
    count[r.kind] += 1;
    pool.push_back(r.a);
    pool.push_back(r.b);
  }
  pending.clear();
}
void Profiler::reset() {
  drain();
  names.clear();
  total_ms.clear();
  count.clear();
}
Profiler::~Profiler() {
  for (Rec &r : pending) { pool.push_back(r.a); pool.push_back(r.b); }
  for (cudaEvent_t e : pool) cudaEventDestroy(e);
}

}  // namespace occu

using namespace occu;

namespace {

occu_status fail(occu_ctx *ctx, occu_status st, const std::string &msg) {
  if (ctx) ctx->err = msg;
  else set_global_error(msg);
  return st;
}

occu_status cuda_fail(occu_ctx *ctx, cudaError_t e, const char *where) {
  return fail(ctx, e == cudaErrorMemoryAllocation ? OCCU_ENOMEM : OCCU_ECUDA,
              std::string(where) + ": " + cudaGetErrorString(e));
}

#define CK(call, where)                                     \
  do {                                                      \
    cudaError_t e__ = (call);                               \
    if (e__ != cudaSuccess) return cuda_fail(ctx, e__, where); \
  } while (0)

#define LK(expr, where)                                                     \
  do {                                                                      \
    int n__ = (expr);                                                       \
    if (n__ < 0) return cuda_fail(ctx, cudaError_t(-n__), where);           \
    ctx->launches += n__;                                                   \
  } while (0)

bool is_device_ptr(const void *p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

occu_status validate_cfg(const occu_config *c) {
  if (!c) return fail(nullptr, OCCU_EINVAL, "config is NULL");
  if (c->L < 1 || c->L > 16) return fail(nullptr, OCCU_EINVAL, "L must be in [1, 16]");
  if (c->d != 64 && c->d != 128 && c->d != 256)
    return fail(nullptr, OCCU_EINVAL, "this build supports d in {64, 128, 256}");
  if (c->d == 256 && (c->msg != OCCU_MSG_CHANNEL_SOFTMAX || c->readout != OCCU_READOUT_MEAN ||
                      c->graphormer != 0 || (c->prec == OCCU_BF16 && c->F_e > 16)))
    return fail(nullptr, OCCU_EINVAL,
                "d = 256 (CTA-pair tensor-core path) supports reading A, the mean readout, no Graphormer layers (OCCU_BF16: F_e <= 16)");
  if (c->F_n < 4 || c->F_n % 4 || c->F_n > 256 || c->F_e < 4 || c->F_e % 4 || c->F_e > 256)
    return fail(nullptr, OCCU_EINVAL, "F_n, F_e must be multiples of 4 in [4, 256]");
  if (c->d_h < 1 || c->d_h > 1024) return fail(nullptr, OCCU_EINVAL, "d_h must be in [1, 1024]");
  if (c->aggr != OCCU_AGGR_SUM && c->aggr != OCCU_AGGR_MEAN)
    return fail(nullptr, OCCU_EINVAL, "aggr must be SUM or MEAN");
  if (c->msg != OCCU_MSG_CHANNEL_SOFTMAX && c->msg != OCCU_MSG_NEIGHBOR_SOFTMAX)
    return fail(nullptr, OCCU_EINVAL, "msg must be CHANNEL_SOFTMAX (reading A) or NEIGHBOR_SOFTMAX (reading B)");
  if (c->msg == OCCU_MSG_NEIGHBOR_SOFTMAX && c->F_n > 128)
    return fail(nullptr, OCCU_EINVAL, "reading B (NEIGHBOR_SOFTMAX) runs on the tensor-core path (F_n <= 128)");
  if (c->prec != OCCU_FP32 && c->prec != OCCU_BF16)
    return fail(nullptr, OCCU_EINVAL, "prec must be OCCU_FP32 or OCCU_BF16");
  if (c->prec == OCCU_BF16 && !(c->F_n <= 128 && (c->F_e <= 16 || c->F_e % 64 == 0)))
    return fail(nullptr, OCCU_EINVAL, "OCCU_BF16 needs F_n <= 128 and F_e <= 16 or a multiple of 64");
  if (!(c->slope > 0.f && c->slope < 1.f)) return fail(nullptr, OCCU_EINVAL, "slope must be in (0,1)");
  if (c->readout != OCCU_READOUT_MEAN && c->readout != OCCU_READOUT_SET_DECODER)
    return fail(nullptr, OCCU_EINVAL, "readout must be MEAN or SET_DECODER");
  if (c->readout == OCCU_READOUT_SET_DECODER) {
    if (c->F_n > 128)
      return fail(nullptr, OCCU_EINVAL, "the Set-Transformer decoder readout runs on the tensor-core path (F_n <= 128)");
    if (c->k < 1 || c->k > 8 || !(c->heads == 1 || c->heads == 2 || c->heads == 4 || c->heads == 8) ||
        c->k * c->heads > 16 || c->d % c->heads)
      return fail(nullptr, OCCU_EINVAL, "decoder: k in [1,8], heads in {1,2,4,8}, k*heads <= 16");
  }
  if (c->graphormer < 0 || c->graphormer > 4)
    return fail(nullptr, OCCU_EINVAL, "graphormer must be in [0, 4]");
  if (c->graphormer > 0) {
    if (c->F_n > 128)
      return fail(nullptr, OCCU_EINVAL, "Graphormer layers run on the tensor-core path (F_n <= 128)");
    if (c->heads < 1 || c->d % c->heads ||
        !(c->d / c->heads == 16 || c->d / c->heads == 32 || c->d / c->heads == 64))
      return fail(nullptr, OCCU_EINVAL, "Graphormer: d / heads must be 16, 32 or 64");
  }
  return OCCU_OK;
}

// Device view of the batch (copies a host batch into `dst` on stream `s`).
occu_status upload_csr(occu_ctx *ctx, const occu_csr_batch *b, DevBuf &dst, cudaStream_t s, DevCsr &out);
occu_status resolve_csr(occu_ctx *ctx, const occu_csr_batch *b, DevCsr &out) {
  return upload_csr(ctx, b, ctx->ws.csr, ctx->stream, out);
}
occu_status upload_csr(occu_ctx *ctx, const occu_csr_batch *b, DevBuf &dst, cudaStream_t s, DevCsr &out) {
  if (!b) return fail(ctx, OCCU_EINVAL, "csr_batch is NULL");
  out.B = b->num_graphs;
  out.N = b->num_nodes;
  out.E = b->num_edges;
  out.max_deg = b->max_in_degree;
  if (b->on_device) {
    out.node_off = b->node_off; out.edge_off = b->edge_off; out.in_ptr = b->in_ptr;
    out.in_src = b->in_src; out.in_dst = b->in_dst; out.in_eid = b->in_eid;
    out.out_ptr = b->out_ptr; out.out_pos = b->out_pos; out.node_graph = b->node_graph;
    return OCCU_OK;
  }
  const size_t B1 = out.B + 1, N1 = out.N + 1, E = out.E, N = out.N;
  const size_t total = 2 * B1 + 2 * N1 + 4 * E + N;
  CK(dst.ensure(total * 4), "csr alloc");
  int32_t *d = dst.as<int32_t>();
  int32_t *q = d;
  const int32_t *srcs[9] = {b->node_off, b->edge_off, b->in_ptr, b->out_ptr, b->in_src,
                            b->in_dst, b->in_eid, b->out_pos, b->node_graph};
  const size_t lens[9] = {B1, B1, N1, N1, E, E, E, E, N};
  const int32_t **dsts[9] = {&out.node_off, &out.edge_off, &out.in_ptr, &out.out_ptr, &out.in_src,
                             &out.in_dst, &out.in_eid, &out.out_pos, &out.node_graph};
  if (b->priv == static_cast<void *>(b->node_off)) {
    // occu_pack output: one contiguous allocation in this order -> a single copy
    CK(cudaMemcpyAsync(d, b->node_off, total * 4, cudaMemcpyHostToDevice, s), "csr H2D");
    for (int i = 0; i < 9; ++i) { *dsts[i] = q; q += lens[i]; }
  } else {
    for (int i = 0; i < 9; ++i) {
      if (lens[i]) CK(cudaMemcpyAsync(q, srcs[i], lens[i] * 4, cudaMemcpyHostToDevice, s), "csr H2D");
      *dsts[i] = q;
      q += lens[i];
    }
  }
  return OCCU_OK;
}

occu_status ensure_layer_bufs(occu_ctx *ctx, const DevCsr &csr) {
  const occu_config &c = ctx->cfg;
  Workspace &w = ctx->ws;
  w.hbar.resize(c.L); w.p.resize(c.L); w.q.resize(c.L); w.e.resize(c.L); w.h.resize(c.L);
  const size_t Nd = size_t(csr.N) * c.d * 4, Ed = size_t(csr.E) * c.d * 4;
  for (int i = 0; i < c.L; ++i) {
    CK(w.hbar[i].ensure(Nd), "alloc hbar");
    CK(w.p[i].ensure(size_t(csr.N) * 4), "alloc p");
    CK(w.q[i].ensure(size_t(csr.N) * 4), "alloc q");
    CK(w.e[i].ensure(Ed), "alloc e");
    CK(w.h[i].ensure(Nd), "alloc h");
  }
  CK(w.g.ensure(Ed), "alloc g");
  CK(w.e0.ensure(size_t(csr.E) * c.F_e * 4), "alloc e0");
  CK(w.r.ensure(size_t(csr.B) * c.d * 4), "alloc r");
  CK(w.c.ensure(size_t(csr.B) * c.d_h * 4), "alloc c");
  CK(w.yhat.ensure(size_t(csr.B) * 4), "alloc yhat");
  return OCCU_OK;
}

// Forward over a device batch; node_feat / edge_feat are device pointers.
occu_status forward(occu_ctx *ctx, const DevCsr &csr, const float *nf, const float *ef,
                    bool save_all) {
  const occu_config &c = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  Workspace &w = ctx->ws;
  occu_status st = ensure_layer_bufs(ctx, csr);
  if (st != OCCU_OK) return st;
  cudaStream_t s = ctx->stream;
  const float *P = ctx->params.as<float>();
  ctx->hbits_layers = 0;
  const bool bf = c.prec == OCCU_BF16;        // kernel path 0 only (occu_set_kernel_path)
  const bool tc = bf || (ctx->path != 1 && tc_supported(c));
  if (!save_all && ctx->path == 0 && ctx->small_enabled && small_forward_ok(ctx, csr)) {
    // CFG1-sized batches: the whole forward in one CTA (kernels_small.cu)
    LK(launch_small_forward(ctx, csr, nf, ef, w.r.as<float>(), w.c.as<float>(), w.yhat.as<float>(), s),
       "small forward");
    ctx->small_fwd = true;
    ctx->h_last_stored = false;
    ctx->last_csr = csr;
    ctx->have_forward = true;
    return OCCU_OK;
  }
  ctx->small_fwd = false;
  // Tensor-core path fusions: a1's edge permutation folded into the layer-1 edge kernel,
  // and the readout's node sums folded into the last aggregation (chunk partials).
  const bool fuse_e0 = tc && c.F_e <= 16;
  const bool dec = c.readout == OCCU_READOUT_SET_DECODER;
  const bool gph = c.graphormer > 0;
  // inference on the fused edge-gate-aggregate kernel: h rows are written by that kernel and
  // its boundary fixup (no readout chunk partials), the last layer's e' is not written at all
  const bool ega = !save_all && !bf && tc && ctx->path == 0 && ctx->fuse_agg &&
                   c.msg == OCCU_MSG_CHANNEL_SOFTMAX && (c.d == 64 || c.d == 128);
  const bool fuse_ro = tc && (bf || ctx->path == 0) && !dec && !gph && !ega;
  if (!fuse_e0) LK(launch_permute_rows(ctx, ef, csr.in_eid, csr.E, c.F_e, w.e0.as<float>(), s), "permute e0");
  if (tc) LK(tc_prepare_weights(ctx, s), "weight images");
  float *rpart = nullptr;
  if (fuse_ro) {
    if (save_all) {
      CK(w.rpart.ensure(size_t(csr.N) * c.d * 4), "alloc rpart");
      rpart = w.rpart.as<float>();
    } else {
      rpart = w.h[c.L - 1].as<float>();     // h_L itself is not stored in this mode
    }
  }
  for (int i = 0; i < c.L; ++i) {
    const bool last = i == c.L - 1;
    FwdLayerArgs a{};
    a.h_in = i == 0 ? nf : w.h[i - 1].as<float>();
    a.K = L.d_in[i];
    a.e_in = i == 0 ? (fuse_e0 ? ef : w.e0.as<float>()) : w.e[i - 1].as<float>();
    a.e_eid = (i == 0 && fuse_e0) ? csr.in_eid : nullptr;
    a.e0_out = (i == 0 && fuse_e0 && save_all) ? w.e0.as<float>() : nullptr;
    a.Ke = L.de_in[i];
    a.W_u = P + L.W_u[i]; a.W_e = P + L.W_e[i]; a.W_m = P + L.W_m[i];
    a.a_s = P + L.a_s[i]; a.a_d = P + L.a_d[i];
    a.hbar = w.hbar[i].as<float>(); a.p = w.p[i].as<float>(); a.q = w.q[i].as<float>();
    a.e_out = (!last || save_all) ? w.e[i].as<float>() : nullptr;
    a.g = w.g.as<float>();
    if (save_all && tc && ctx->path == 0) {    // the backward reads the gates (no recompute)
      if (w.gs.size() < size_t(c.L)) w.gs.resize(c.L);
      CK(w.gs[i].ensure(size_t(csr.E) * c.d * (bf ? 2 : 4)), "alloc saved gates");
      a.g = w.gs[i].as<float>();
    }
    a.h_out = w.h[i].as<float>();
    a.save_w = save_all && c.msg == OCCU_MSG_NEIGHBOR_SOFTMAX;   // reading B: weights for the backward
    if (save_all && tc && ctx->path == 0 && c.msg == OCCU_MSG_CHANNEL_SOFTMAX) {
      // sign bits of h^i: the backward's LReLU'(h^i) mask of dh^i (dh_prev of layer i+1; the
      // head backward's broadcast for i = L-1)
      if (w.hbits.size() < size_t(c.L)) w.hbits.resize(c.L);
      CK(w.hbits[i].ensure(size_t(csr.N) * (c.d / 32) * 4), "alloc h sign bits");
      a.h_bits = reinterpret_cast<uint32_t *>(w.hbits[i].ptr);
      ctx->hbits_layers = i + 1;
    }
    a.infer = ega;
    if (tc) {
      a.e_out = (ega && last) ? nullptr : w.e[i].as<float>();   // the gate kernel re-reads e'
      if (last && fuse_ro) {
        a.rpart = rpart;
        if (!save_all) a.h_out = nullptr;
      }
      if (bf) {
        LK(launch_forward_layer_bf16(ctx, csr, i, a, s), "forward layer (bf16)");
        continue;
      }
      CK(w.tcpart.ensure(tc_partial_floats(csr.E, c.d) * 4), "alloc tc partials");
      LK(launch_forward_layer_tc(ctx, csr, i, a, w.tcpart.as<float>(), s), "forward layer (tc)");
    } else {
      LK(launch_forward_layer(ctx, csr, a, s), "forward layer");
    }
  }
  const float *h_top = w.h[c.L - 1].as<float>();
  if (bf && (gph || dec)) {
    // R41: in OCCU_BF16 the Graphormer layers / the decoder run in FP32 on the BF16-stored h_L
    CK(w.hf.ensure(size_t(csr.N) * c.d * 4), "alloc FP32 h_L");
    LK(launch_bf16_to_f32(ctx, w.h[c.L - 1].ptr, size_t(csr.N) * c.d, w.hf.as<float>(), s), "h_L to FP32");
    h_top = w.hf.as<float>();
  }
  if (gph) {
    // NEXT-3: Graphormer layers over each graph's node set (ping-pong between two buffers)
    if (w.gh.size() < size_t(c.graphormer)) w.gh.resize(c.graphormer);
    for (int j = 0; j < c.graphormer; ++j) CK(w.gh[j].ensure(size_t(csr.N) * c.d * 4), "alloc graphormer states");
    CK(w.gx.ensure(size_t(csr.N) * c.d * 4), "alloc graphormer scratch");
    CK(w.gqkv.ensure(size_t(csr.N) * 3 * c.d * 4), "alloc graphormer scratch");
    CK(w.go.ensure(size_t(csr.N) * c.d * 4), "alloc graphormer scratch");
    if (save_all) {                     // training: every intermediate kept for the backward
      if (w.gsave.size() < size_t(8 * c.graphormer)) w.gsave.resize(8 * c.graphormer);
      for (auto &b : w.gsave) CK(b.ensure(size_t(csr.N) * c.d * 4), "alloc graphormer saves");
    }
    for (int j = 0; j < c.graphormer; ++j) {
      float *out = w.gh[j].as<float>();
      GphSave sv;
      if (save_all) {
        float **f[8] = {&sv.X1, &sv.Q, &sv.K, &sv.V, &sv.O, &sv.Hb, &sv.X2, &sv.T};
        for (int t = 0; t < 8; ++t) *f[t] = w.gsave[8 * j + t].as<float>();
      }
      LK(launch_graphormer_layer(ctx, csr, j, h_top, out, w.gx.as<float>(), w.gqkv.as<float>(),
                                 w.go.as<float>(), s, save_all ? &sv : nullptr),
         "graphormer layer");
      h_top = out;
    }
  }
  if (dec) {
    // NEXT-2: Set-Transformer decoder per graph, head on the flattened k·d output
    CK(w.dT.ensure(size_t(csr.N) * c.d * 4), "alloc decoder scratch");
    CK(w.dZ.ensure(size_t(csr.N) * c.d * 4), "alloc decoder scratch");
    CK(w.r.ensure(size_t(csr.B) * c.k * c.d * 4), "alloc r");
    LK(launch_set_decoder(ctx, csr, h_top, w.dT.as<float>(), w.dZ.as<float>(),
                          w.r.as<float>(), w.c.as<float>(), w.yhat.as<float>(), s),
       "set decoder");
  } else {
    LK(launch_readout_head(ctx, csr, fuse_ro ? rpart : h_top, fuse_ro, P,
                           w.r.as<float>(), w.c.as<float>(), w.yhat.as<float>(), s),
       "readout/head");
  }
  ctx->h_last_stored = !fuse_ro || save_all;
  ctx->last_csr = csr;
  ctx->have_forward = true;
  return OCCU_OK;
}

struct Staged {
  const float *nf = nullptr, *ef = nullptr, *y = nullptr;
  bool host = false;
};

occu_status stage_inputs(occu_ctx *ctx, const DevCsr &csr, const float *nf, const float *ef,
                         const float *y, Staged &out) {
  const occu_config &c = ctx->cfg;
  if (!nf || (csr.E > 0 && !ef)) return fail(ctx, OCCU_EINVAL, "feature pointer is NULL");
  out.host = !is_device_ptr(nf);
  if (!out.host) {
    out.nf = nf; out.ef = ef; out.y = y;
    return OCCU_OK;
  }
  Workspace &w = ctx->ws;
  CK(w.node_feat.ensure(size_t(csr.N) * c.F_n * 4), "alloc node_feat");
  CK(w.edge_feat.ensure(size_t(csr.E) * c.F_e * 4), "alloc edge_feat");
  CK(cudaMemcpyAsync(w.node_feat.ptr, nf, size_t(csr.N) * c.F_n * 4, cudaMemcpyHostToDevice,
                     ctx->stream), "node_feat H2D");
  if (csr.E > 0)
    CK(cudaMemcpyAsync(w.edge_feat.ptr, ef, size_t(csr.E) * c.F_e * 4, cudaMemcpyHostToDevice,
                       ctx->stream), "edge_feat H2D");
  out.nf = w.node_feat.as<float>();
  out.ef = w.edge_feat.as<float>();
  if (y) {
    CK(w.targets.ensure(size_t(csr.B) * 4), "alloc targets");
    CK(cudaMemcpyAsync(w.targets.ptr, y, size_t(csr.B) * 4, cudaMemcpyHostToDevice, ctx->stream),
       "targets H2D");
    out.y = w.targets.as<float>();
  }
  return OCCU_OK;
}

occu_status check_ready(occu_ctx *ctx) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  if (!ctx->weights_ready) return fail(ctx, OCCU_ENOTREADY, "weights not initialised");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  return OCCU_OK;
}

occu_status check_train(occu_ctx *ctx, const occu_batch *batch, const float *targets) {
  occu_status st = check_ready(ctx);
  if (st != OCCU_OK) return st;
  if (!batch || !batch->csr || !targets) return fail(ctx, OCCU_EINVAL, "batch/targets NULL");
  if (batch->global_num_graphs < batch->csr->num_graphs)
    return fail(ctx, OCCU_EINVAL, "global_num_graphs < local num_graphs");
  const bool stack = ctx->cfg.readout == OCCU_READOUT_SET_DECODER || ctx->cfg.graphormer > 0;
  if (stack && (ctx->cfg.prec != OCCU_FP32 || ctx->path != 0))
    return fail(ctx, OCCU_EINVAL, "training through the Graphormer layers / decoder readout runs in OCCU_FP32 on kernel path 0");
  if (ctx->cfg.msg == OCCU_MSG_NEIGHBOR_SOFTMAX && ctx->cfg.prec == OCCU_BF16)
    return fail(ctx, OCCU_EINVAL, "reading B in OCCU_BF16 is inference-only in this build");
  if (ctx->cfg.d > 128)
    return fail(ctx, OCCU_EINVAL, "d = 256 is inference-only in this build");
  return OCCU_OK;
}

// Forward with saves + backward of a batch already on the device (csr, stg device pointers);
// gradients (+ the loss in slot `total`) land in ctx->grads.
occu_status grads_core(occu_ctx *ctx, const DevCsr &csr, const Staged &stg, int32_t global_B) {
  occu_status st;
  const bool stack = ctx->cfg.readout == OCCU_READOUT_SET_DECODER || ctx->cfg.graphormer > 0;
  if ((st = forward(ctx, csr, stg.nf, stg.ef, true)) != OCCU_OK) return st;
  const occu_config &c = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  Workspace &w = ctx->ws;
  const size_t Nd = size_t(csr.N) * c.d * 4, Ed = size_t(csr.E) * c.d * 4;
  CK(w.dy.ensure(size_t(csr.B) * 4), "alloc");
  CK(w.dc.ensure(size_t(csr.B) * c.d_h * 4), "alloc");
  CK(w.dr.ensure(size_t(csr.B) * L.head_in * 4), "alloc");
  CK(w.dh.ensure(Nd), "alloc");
  CK(w.dP.ensure(Nd), "alloc");
  CK(w.MG.ensure(Ed), "alloc");
  CK(w.DV.ensure(Ed), "alloc");
  CK(w.DZ.ensure(Ed), "alloc");
  CK(w.deA.ensure(Ed), "alloc");
  CK(w.deB.ensure(Ed), "alloc");
  CK(w.dalpha.ensure(size_t(csr.E) * 4), "alloc");
  CK(w.dpq.ensure(size_t(csr.N) * 8), "alloc");
  CK(w.loss.ensure(4), "alloc");
  cudaStream_t s = ctx->stream;
  LK(launch_head_backward(ctx, csr, stg.y, global_B, s), "head backward");
  if (stack) {
    // NEXT-2 / NEXT-3 training: ∂L/∂(stack top) from the readout, then the Graphormer layers in
    // reverse, then dA of the last ANEE layer (what the ANEE backward consumes in w.dh)
    for (auto &b : w.gdh) CK(b.ensure(Nd), "alloc stack gradients");
    const size_t scr = 5 * Nd + size_t(csr.N) * std::max(c.heads, 1) * 16;
    CK(w.gscr.ensure(scr), "alloc stack scratch");
    float *g = w.gdh[0].as<float>();
    const float *top = c.graphormer > 0 ? w.gh[c.graphormer - 1].as<float>() : w.h[c.L - 1].as<float>();
    if (c.readout == OCCU_READOUT_SET_DECODER) {
      // NEXT-2: decoder backward from dr down to its node-state input (the stack top)
      float *scr = w.gscr.as<float>();
      LK(launch_set_decoder_bwd(ctx, csr, top, w.dT.as<float>(), w.dZ.as<float>(), w.dr.as<float>(),
                                scr, scr + size_t(csr.N) * c.d, g, s),
         "decoder backward");
    } else {
      // mean readout: broadcast_dh (launched by the head backward without a mask) left dr/n_b
      CK(cudaMemcpyAsync(g, w.dh.ptr, Nd, cudaMemcpyDeviceToDevice, s), "copy dh");
    }
    for (int j = c.graphormer - 1; j >= 0; --j) {
      const float *hin = j == 0 ? w.h[c.L - 1].as<float>() : w.gh[j - 1].as<float>();
      GphSave sv;
      float **f[8] = {&sv.X1, &sv.Q, &sv.K, &sv.V, &sv.O, &sv.Hb, &sv.X2, &sv.T};
      for (int t = 0; t < 8; ++t) *f[t] = w.gsave[8 * j + t].as<float>();
      float *gout = w.gdh[(c.graphormer - j) & 1].as<float>();
      LK(launch_graphormer_layer_bwd(ctx, csr, j, hin, sv, g, gout, w.gscr.as<float>(), s),
         "graphormer backward");
      g = gout;
    }
    LK(launch_mask_dA(ctx, csr, g, w.h[c.L - 1].as<float>(), w.dh.as<float>(), s), "mask dA");
  }
  for (int i = c.L - 1; i >= 0; --i) {
    BwdLayerArgs a{};
    a.layer = i;
    a.h_in = i == 0 ? stg.nf : w.h[i - 1].as<float>();
    a.K = L.d_in[i];
    a.e_in = i == 0 ? w.e0.as<float>() : w.e[i - 1].as<float>();
    a.Ke = L.de_in[i];
    a.hbar = w.hbar[i].as<float>(); a.p = w.p[i].as<float>(); a.q = w.q[i].as<float>();
    a.e = w.e[i].as<float>(); a.h = w.h[i].as<float>();
    a.g = (ctx->path == 0 && w.gs.size() > size_t(i)) ? w.gs[i].as<float>() : nullptr;
    a.dh = w.dh.as<float>();
    a.de_out = i < c.L - 1 ? w.deB.as<float>() : nullptr;
    a.de_prev = i > 0 ? w.deB.as<float>() : nullptr;     // read-before-write ordering, see DESIGN
    a.dh_prev = i > 0 ? w.dh.as<float>() : nullptr;
    if (i > 0 && ctx->hbits_layers >= i) a.h_in_bits = reinterpret_cast<const uint32_t *>(w.hbits[i - 1].ptr);
    a.bf = c.prec == OCCU_BF16;     // h̄, e', g, h (and h_in, e_in for i > 0) stored as BF16
    LK(launch_backward_layer(ctx, csr, a, s), "backward layer");
  }
  // loss rides along the gradient buffer (slot `total`) so one allreduce sums both
  CK(cudaMemcpyAsync(ctx->grads.as<float>() + L.total, w.loss.ptr, 4, cudaMemcpyDeviceToDevice, s),
     "loss copy");
  return OCCU_OK;
}

occu_status grads_impl(occu_ctx *ctx, const occu_batch *batch, const float *targets, Staged &stg,
                       DevCsr &csr) {
  occu_status st = check_train(ctx, batch, targets);
  if (st != OCCU_OK) return st;
  ctx->launches = 0;
  if ((st = resolve_csr(ctx, batch->csr, csr)) != OCCU_OK) return st;
  if ((st = stage_inputs(ctx, csr, batch->node_feat, batch->edge_feat, targets, stg)) != OCCU_OK)
    return st;
  return grads_core(ctx, csr, stg, batch->global_num_graphs);
}

// ---- NCCL watchdog -------------------------------------------------------------------
// The communicator is non-blocking (ncclConfig_t::blocking = 0): NCCL calls return at once
// (possibly ncclInProgress) and progress / asynchronous errors are polled here, so a dead
// peer or a stuck collective surfaces as OCCU_ENCCL after ctx->nccl_timeout_s instead of a
// hang; the communicator is then aborted (ncclCommAbort) and dropped.
double now_s() {
  timespec t;
  clock_gettime(CLOCK_MONOTONIC, &t);
  return double(t.tv_sec) + 1e-9 * double(t.tv_nsec);
}

occu_status nccl_abort(occu_ctx *ctx, const std::string &why) {
  if (ctx->comm) {
    ncclCommAbort(ctx->comm);
    ctx->comm = nullptr;
  }
  ctx->comm_aborted = true;
  return fail(ctx, OCCU_ENCCL, why);
}

// Wait until the communicator has no NCCL call in progress (setup or an enqueue).
occu_status nccl_settle(occu_ctx *ctx, const char *what) {
  const double t0 = now_s();
  for (;;) {
    ncclResult_t st = ncclSuccess;
    ncclResult_t r = ncclCommGetAsyncError(ctx->comm, &st);
    if (r != ncclSuccess) return nccl_abort(ctx, std::string(what) + ": ncclCommGetAsyncError: " + ncclGetErrorString(r));
    if (st == ncclSuccess) return OCCU_OK;
    if (st != ncclInProgress) return nccl_abort(ctx, std::string(what) + ": " + ncclGetErrorString(st));
    if (ctx->nccl_timeout_s > 0 && now_s() - t0 > ctx->nccl_timeout_s)
      return nccl_abort(ctx, std::string(what) + ": timed out (ncclCommAbort)");
    sched_yield();
  }
}

// Host wait for the ctx stream; with a communicator, poll NCCL errors and the timeout.
occu_status stream_wait(occu_ctx *ctx, const char *what) {
  if (!ctx->comm) {
    CK(cudaStreamSynchronize(ctx->stream), what);
    return OCCU_OK;
  }
  const double t0 = now_s();
  for (;;) {
    cudaError_t e = cudaStreamQuery(ctx->stream);
    if (e == cudaSuccess) return OCCU_OK;
    if (e != cudaErrorNotReady) return cuda_fail(ctx, e, what);
    ncclResult_t st = ncclSuccess;
    if (ncclCommGetAsyncError(ctx->comm, &st) != ncclSuccess || (st != ncclSuccess && st != ncclInProgress))
      return nccl_abort(ctx, std::string(what) + ": NCCL asynchronous error " + ncclGetErrorString(st));
    if (ctx->nccl_timeout_s > 0 && now_s() - t0 > ctx->nccl_timeout_s)
      return nccl_abort(ctx, std::string(what) + ": no progress within the timeout (ncclCommAbort)");
    usleep(20);
  }
}

// a11 + a12 after the backward: the NCCL allreduce (when a communicator exists), then Adam.
occu_status allreduce_adam(occu_ctx *ctx, float lr) {
  occu_status st;
  const size_t n = ctx->layout.total + 1;
  if (ctx->comm_aborted && !ctx->comm)
    return fail(ctx, OCCU_ENCCL, "the communicator was aborted; call occu_dist_init again");
  if (ctx->comm) {
    // a11: sum of the flat gradient (+ loss slot) over the ranks, in place, on the ctx stream
    ncclResult_t r = ncclAllReduce(ctx->grads.ptr, ctx->grads.ptr, n, ncclFloat32, ncclSum,
                                   ctx->comm, ctx->stream);
    if (r != ncclSuccess && r != ncclInProgress)
      return nccl_abort(ctx, std::string("ncclAllReduce: ") + ncclGetErrorString(r));
    if ((st = nccl_settle(ctx, "ncclAllReduce")) != OCCU_OK) return st;
  }
  ctx->adam_t += 1;
  LK(launch_adam(ctx, lr, ctx->stream), "adam");
  return OCCU_OK;
}

}  // namespace

// ============================================================================
extern "C" {

size_t occu_num_params(const occu_config *cfg) {
  if (!cfg) return 0;
  return make_layout(*cfg).total;
}

occu_status occu_create(occu_ctx **out, const occu_config *cfg, int cuda_device, void *cuda_stream) {
  if (!out) return fail(nullptr, OCCU_EINVAL, "out is NULL");
  *out = nullptr;
  occu_status st = validate_cfg(cfg);
  if (st != OCCU_OK) return st;
  cudaError_t e = cudaSetDevice(cuda_device);
  if (e != cudaSuccess) return fail(nullptr, OCCU_ECUDA, std::string("cudaSetDevice: ") + cudaGetErrorString(e));
  occu_ctx *ctx = new (std::nothrow) occu_ctx();
  if (!ctx) return OCCU_ENOMEM;
  ctx->cfg = *cfg;
  ctx->layout = make_layout(*cfg);
  ctx->device = cuda_device;
  ctx->stream = static_cast<cudaStream_t>(cuda_stream);
  cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
  if (const char *e = getenv("OCCU_L2_ORDER")) ctx->l2_order = atoi(e);   // A/B switches
  if (const char *e = getenv("OCCU_FUSE_EG")) ctx->fuse_edge_gate = atoi(e);
  if (const char *e = getenv("OCCU_FUSE_EGA")) ctx->fuse_agg = atoi(e);
  if (const char *e = getenv("OCCU_PDL")) ctx->pdl = atoi(e);
  const size_t pb = (ctx->layout.total + 1) * 4;
  if (ctx->params.ensure(pb) != cudaSuccess || ctx->grads.ensure(pb) != cudaSuccess ||
      ctx->adam_m.ensure(pb) != cudaSuccess || ctx->adam_v.ensure(pb) != cudaSuccess) {
    delete ctx;
    return fail(nullptr, OCCU_ENOMEM, "parameter allocation failed");
  }
  cudaMemset(ctx->grads.ptr, 0, pb);
  cudaMemset(ctx->adam_m.ptr, 0, pb);
  cudaMemset(ctx->adam_v.ptr, 0, pb);
  *out = ctx;
  return OCCU_OK;
}

occu_status occu_destroy(occu_ctx *ctx) {
  if (!ctx) return OCCU_OK;
  cudaSetDevice(ctx->device);
  cudaStreamSynchronize(ctx->stream);
  if (ctx->comm) ncclCommDestroy(ctx->comm);
  if (ctx->copy_stream) {
    cudaStreamSynchronize(ctx->copy_stream);
    cudaStreamDestroy(ctx->copy_stream);
    for (int k = 0; k < 2; ++k) {
      cudaEventDestroy(ctx->a_copied[k]);
      cudaEventDestroy(ctx->a_free[k]);
    }
  }
  ctx->ws.release_all();
  ctx->params.release();
  ctx->wimg.release();
  ctx->wjobs.release();
  ctx->wfexp.release();
  ctx->grads.release();
  ctx->adam_m.release();
  ctx->adam_v.release();
  delete ctx;
  return OCCU_OK;
}

occu_status occu_set_stream(occu_ctx *ctx, void *cuda_stream) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  ctx->stream = static_cast<cudaStream_t>(cuda_stream);
  return OCCU_OK;
}

occu_status occu_set_params(occu_ctx *ctx, const float *host_flat, size_t n) {
  if (!ctx || !host_flat) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (n != ctx->layout.total) return fail(ctx, OCCU_EINVAL, "parameter count mismatch");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(cudaMemcpyAsync(ctx->params.ptr, host_flat, n * 4, cudaMemcpyHostToDevice, ctx->stream), "H2D");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  ctx->weights_ready = true;
  ctx->params_version += 1;
  return OCCU_OK;
}

occu_status occu_get_params(const occu_ctx *cctx, float *host_flat, size_t n) {
  occu_ctx *ctx = const_cast<occu_ctx *>(cctx);
  if (!ctx || !host_flat) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (n != ctx->layout.total) return fail(ctx, OCCU_EINVAL, "parameter count mismatch");
  if (!ctx->weights_ready) return fail(ctx, OCCU_ENOTREADY, "weights not initialised");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(cudaMemcpyAsync(host_flat, ctx->params.ptr, n * 4, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  return OCCU_OK;
}

occu_status occu_init_weights(occu_ctx *ctx, uint64_t seed) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  std::vector<float> w;
  init_flat(ctx->cfg, seed, w);
  return occu_set_params(ctx, w.data(), w.size());
}

occu_status occu_load_weights(occu_ctx *ctx, const char *path) {
  if (!ctx || !path) return fail(ctx, OCCU_EINVAL, "NULL argument");
  std::vector<unsigned char> payload;
  std::string err;
  occu_status st = read_file(path, "OCCUW001", ctx->cfg, payload, ctx->layout.total * 4, err);
  if (st != OCCU_OK) return fail(ctx, st, "occu_load_weights: " + err);
  return occu_set_params(ctx, reinterpret_cast<const float *>(payload.data()), ctx->layout.total);
}

occu_status occu_save_weights(const occu_ctx *cctx, const char *path) {
  occu_ctx *ctx = const_cast<occu_ctx *>(cctx);
  if (!ctx || !path) return fail(ctx, OCCU_EINVAL, "NULL argument");
  std::vector<float> w(ctx->layout.total);
  occu_status st = occu_get_params(ctx, w.data(), w.size());
  if (st != OCCU_OK) return st;
  std::string err;
  if (!write_file(path, "OCCUW001", ctx->cfg, {{w.data(), w.size() * 4}}, err))
    return fail(ctx, OCCU_EINVAL, err);
  return OCCU_OK;
}

occu_status occu_batch_to_device(occu_ctx *ctx, const occu_csr_batch *host, occu_csr_batch **dev_out) {
  if (!ctx || !host || !dev_out) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (host->on_device) return fail(ctx, OCCU_EINVAL, "batch already on device");
  *dev_out = nullptr;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  const size_t B1 = host->num_graphs + 1, N1 = host->num_nodes + 1, E = host->num_edges,
               N = host->num_nodes;
  const size_t total = 2 * B1 + 2 * N1 + 4 * E + N;
  int32_t *d = nullptr;
  CK(cudaMalloc(&d, std::max<size_t>(total, 1) * 4), "batch alloc");
  cudaError_t e = cudaMemcpyAsync(d, host->node_off, total * 4, cudaMemcpyHostToDevice, ctx->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
  if (e != cudaSuccess) {
    cudaFree(d);
    return cuda_fail(ctx, e, "batch H2D");
  }
  occu_csr_batch *b = static_cast<occu_csr_batch *>(calloc(1, sizeof(occu_csr_batch)));
  if (!b) {
    cudaFree(d);
    return OCCU_ENOMEM;
  }
  *b = *host;
  int32_t *q = d;
  b->node_off = q; q += B1;
  b->edge_off = q; q += B1;
  b->in_ptr = q; q += N1;
  b->out_ptr = q; q += N1;
  b->in_src = q; q += E;
  b->in_dst = q; q += E;
  b->in_eid = q; q += E;
  b->out_pos = q; q += E;
  b->node_graph = q;
  b->on_device = 1;
  b->priv = d;
  *dev_out = b;
  return OCCU_OK;
}

void occu_batch_free(occu_csr_batch *b) {
  if (!b) return;
  if (b->on_device) {
    cudaFree(b->priv);
    free(b);
  } else {
    occu_host_batch_release(b);
  }
}

occu_status occu_predict(occu_ctx *ctx, const occu_csr_batch *csr_batch, const float *node_feat,
                         const float *edge_feat, float *out_occ) {
  occu_status st = check_ready(ctx);
  if (st != OCCU_OK) return st;
  if (!out_occ) return fail(ctx, OCCU_EINVAL, "out_occ is NULL");
  ctx->launches = 0;
  DevCsr csr;
  if ((st = resolve_csr(ctx, csr_batch, csr)) != OCCU_OK) return st;
  Staged stg;
  if ((st = stage_inputs(ctx, csr, node_feat, edge_feat, nullptr, stg)) != OCCU_OK) return st;
  if (stg.host == is_device_ptr(out_occ))
    return fail(ctx, OCCU_EINVAL, "out_occ must be in the same memory space as the features");
  if ((st = forward(ctx, csr, stg.nf, stg.ef, ctx->keep)) != OCCU_OK) return st;
  const size_t ob = size_t(csr.B) * 4;
  if (stg.host) {
    CK(cudaMemcpyAsync(out_occ, ctx->ws.yhat.ptr, ob, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
    CK(cudaStreamSynchronize(ctx->stream), "sync");
  } else {
    CK(cudaMemcpyAsync(out_occ, ctx->ws.yhat.ptr, ob, cudaMemcpyDeviceToDevice, ctx->stream), "D2D");
  }
  CK(cudaGetLastError(), "predict");
  return OCCU_OK;
}

occu_status occu_predict_async(occu_ctx *ctx, const occu_csr_batch *csr_batch,
                               const float *node_feat, const float *edge_feat, float *out_occ) {
  occu_status st = check_ready(ctx);
  if (st != OCCU_OK) return st;
  if (!csr_batch || !node_feat || !out_occ || (csr_batch->num_edges > 0 && !edge_feat))
    return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (csr_batch->on_device || is_device_ptr(node_feat) || is_device_ptr(out_occ))
    return fail(ctx, OCCU_EINVAL, "occu_predict_async takes a host batch and host (pinned) buffers");
  if (!ctx->copy_stream) {
    CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking), "copy stream");
    for (int k = 0; k < 2; ++k) {
      CK(cudaEventCreateWithFlags(&ctx->a_copied[k], cudaEventDisableTiming), "event");
      CK(cudaEventCreateWithFlags(&ctx->a_free[k], cudaEventDisableTiming), "event");
    }
  }
  ctx->launches = 0;
  const int slot = ctx->a_slot;
  ctx->a_slot ^= 1;
  // the previous call's host inputs become reusable once its copy has landed: the host
  // waits here (the copy is the pipeline's slowest stage, so this costs no throughput)
  CK(cudaEventSynchronize(ctx->a_copied[slot ^ 1]), "wait previous copy");
  const occu_config &c = ctx->cfg;
  Workspace &w = ctx->ws;
  // the slot's buffers are reused only after the forward that read them has finished
  CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->a_free[slot], 0), "wait slot");
  DevCsr csr;
  if ((st = upload_csr(ctx, csr_batch, w.acsr[slot], ctx->copy_stream, csr)) != OCCU_OK) return st;
  CK(w.anf[slot].ensure(size_t(csr.N) * c.F_n * 4), "alloc node_feat");
  CK(w.aef[slot].ensure(std::max<size_t>(size_t(csr.E) * c.F_e * 4, 4)), "alloc edge_feat");
  CK(cudaMemcpyAsync(w.anf[slot].ptr, node_feat, size_t(csr.N) * c.F_n * 4, cudaMemcpyHostToDevice,
                     ctx->copy_stream), "node_feat H2D");
  if (csr.E > 0)
    CK(cudaMemcpyAsync(w.aef[slot].ptr, edge_feat, size_t(csr.E) * c.F_e * 4, cudaMemcpyHostToDevice,
                       ctx->copy_stream), "edge_feat H2D");
  CK(cudaEventRecord(ctx->a_copied[slot], ctx->copy_stream), "record");
  CK(cudaStreamWaitEvent(ctx->stream, ctx->a_copied[slot], 0), "wait copy");
  if ((st = forward(ctx, csr, w.anf[slot].as<float>(), w.aef[slot].as<float>(), ctx->keep)) != OCCU_OK)
    return st;
  CK(cudaEventRecord(ctx->a_free[slot], ctx->stream), "record");
  CK(cudaMemcpyAsync(out_occ, w.yhat.ptr, size_t(csr.B) * 4, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
  CK(cudaGetLastError(), "predict_async");
  return OCCU_OK;
}

occu_status occu_wait(occu_ctx *ctx) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  if (ctx->copy_stream) CK(cudaStreamSynchronize(ctx->copy_stream), "sync");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  return OCCU_OK;
}

occu_status occu_compute_grads(occu_ctx *ctx, const occu_batch *batch, const float *targets,
                               float *out_loss) {
  Staged stg;
  DevCsr csr;
  occu_status st = grads_impl(ctx, batch, targets, stg, csr);
  if (st != OCCU_OK) return st;
  if (out_loss || stg.host) {
    float l = 0.f;
    CK(cudaMemcpyAsync(&l, ctx->grads.as<float>() + ctx->layout.total, 4, cudaMemcpyDeviceToHost,
                       ctx->stream), "loss D2H");
    CK(cudaStreamSynchronize(ctx->stream), "sync");
    if (out_loss) *out_loss = l;
  }
  return OCCU_OK;
}

occu_status occu_train_step(occu_ctx *ctx, const occu_batch *batch, const float *targets,
                            float lr, float *out_loss) {
  Staged stg;
  DevCsr csr;
  occu_status st = grads_impl(ctx, batch, targets, stg, csr);
  if (st != OCCU_OK) return st;
  if ((st = allreduce_adam(ctx, lr)) != OCCU_OK) return st;
  if (out_loss || stg.host) {
    float l = 0.f;
    CK(cudaMemcpyAsync(&l, ctx->grads.as<float>() + ctx->layout.total, 4, cudaMemcpyDeviceToHost,
                       ctx->stream), "loss D2H");
    if ((st = stream_wait(ctx, "train step")) != OCCU_OK) return st;
    if (out_loss) *out_loss = l;
  }
  return OCCU_OK;
}

occu_status occu_train_step_async(occu_ctx *ctx, const occu_batch *batch, const float *targets,
                                  float lr, float *out_loss) {
  occu_status st = check_train(ctx, batch, targets);
  if (st != OCCU_OK) return st;
  const occu_csr_batch *hb = batch->csr;
  if (hb->on_device || !batch->node_feat || is_device_ptr(batch->node_feat) || is_device_ptr(targets) ||
      (out_loss && is_device_ptr(out_loss)) || (hb->num_edges > 0 && !batch->edge_feat))
    return fail(ctx, OCCU_EINVAL, "occu_train_step_async takes a host batch and host (pinned) buffers");
  if (!ctx->copy_stream) {
    CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking), "copy stream");
    for (int k = 0; k < 2; ++k) {
      CK(cudaEventCreateWithFlags(&ctx->a_copied[k], cudaEventDisableTiming), "event");
      CK(cudaEventCreateWithFlags(&ctx->a_free[k], cudaEventDisableTiming), "event");
    }
  }
  ctx->launches = 0;
  const int slot = ctx->a_slot;
  ctx->a_slot ^= 1;
  // the previous call's host inputs become reusable once its copies have landed
  CK(cudaEventSynchronize(ctx->a_copied[slot ^ 1]), "wait previous copy");
  const occu_config &c = ctx->cfg;
  Workspace &w = ctx->ws;
  // the slot's buffers are reused only after the step that read them has finished
  CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->a_free[slot], 0), "wait slot");
  DevCsr csr;
  if ((st = upload_csr(ctx, hb, w.acsr[slot], ctx->copy_stream, csr)) != OCCU_OK) return st;
  CK(w.anf[slot].ensure(size_t(csr.N) * c.F_n * 4), "alloc node_feat");
  CK(w.aef[slot].ensure(std::max<size_t>(size_t(csr.E) * c.F_e * 4, 4)), "alloc edge_feat");
  CK(w.aty[slot].ensure(size_t(csr.B) * 4), "alloc targets");
  CK(cudaMemcpyAsync(w.anf[slot].ptr, batch->node_feat, size_t(csr.N) * c.F_n * 4,
                     cudaMemcpyHostToDevice, ctx->copy_stream), "node_feat H2D");
  if (csr.E > 0)
    CK(cudaMemcpyAsync(w.aef[slot].ptr, batch->edge_feat, size_t(csr.E) * c.F_e * 4,
                       cudaMemcpyHostToDevice, ctx->copy_stream), "edge_feat H2D");
  CK(cudaMemcpyAsync(w.aty[slot].ptr, targets, size_t(csr.B) * 4, cudaMemcpyHostToDevice,
                     ctx->copy_stream), "targets H2D");
  CK(cudaEventRecord(ctx->a_copied[slot], ctx->copy_stream), "record");
  CK(cudaStreamWaitEvent(ctx->stream, ctx->a_copied[slot], 0), "wait copy");
  Staged stg;
  stg.nf = w.anf[slot].as<float>();
  stg.ef = w.aef[slot].as<float>();
  stg.y = w.aty[slot].as<float>();
  stg.host = false;
  if ((st = grads_core(ctx, csr, stg, batch->global_num_graphs)) != OCCU_OK) return st;
  if ((st = allreduce_adam(ctx, lr)) != OCCU_OK) return st;
  CK(cudaEventRecord(ctx->a_free[slot], ctx->stream), "record");
  if (out_loss)
    CK(cudaMemcpyAsync(out_loss, ctx->grads.as<float>() + ctx->layout.total, 4,
                       cudaMemcpyDeviceToHost, ctx->stream), "loss D2H");
  CK(cudaGetLastError(), "train_step_async");
  return OCCU_OK;
}

occu_status occu_get_grads(const occu_ctx *cctx, float *host_flat, size_t n) {
  occu_ctx *ctx = const_cast<occu_ctx *>(cctx);
  if (!ctx || !host_flat) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (n != ctx->layout.total) return fail(ctx, OCCU_EINVAL, "parameter count mismatch");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(cudaMemcpyAsync(host_flat, ctx->grads.ptr, n * 4, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  return OCCU_OK;
}

occu_status occu_test_wgrad(occu_ctx *ctx, const float *X, int32_t A, const void *Y, int32_t Bn,
                            int64_t R, int32_t y_bf16, float *out) {
  if (!ctx || !X || !Y || !out) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (A < 1 || Bn < 1 || R < 0 || A > 128 || Bn > 128) return fail(ctx, OCCU_EINVAL, "bad shape");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->launches = 0;
  LK(launch_wgrad(ctx, X, A, Y, Bn, long(R), out, ctx->stream, y_bf16 != 0), "wgrad");
  return OCCU_OK;
}

occu_status occu_set_weight_decay(occu_ctx *ctx, float wd) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  if (!(wd >= 0.f)) return fail(ctx, OCCU_EINVAL, "weight decay must be >= 0");
  ctx->weight_decay = wd;
  return OCCU_OK;
}

occu_status occu_nccl_unique_id(void *out_128_bytes) {
  if (!out_128_bytes) return fail(nullptr, OCCU_EINVAL, "NULL argument");
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return fail(nullptr, OCCU_ENCCL, std::string("ncclGetUniqueId: ") + ncclGetErrorString(r));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  memcpy(out_128_bytes, &id, 128);
  return OCCU_OK;
}

occu_status occu_dist_init(occu_ctx *ctx, int rank, int world, const void *nccl_unique_id) {
  if (!ctx || !nccl_unique_id) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (world < 1 || rank < 0 || rank >= world) return fail(ctx, OCCU_EINVAL, "bad rank/world");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  if (ctx->comm) {
    ncclCommDestroy(ctx->comm);
    ctx->comm = nullptr;
  }
  ncclUniqueId id;
  memcpy(&id, nccl_unique_id, 128);
  ncclConfig_t cfg = NCCL_CONFIG_INITIALIZER;
  cfg.blocking = 0;                      // progress polled by the watchdog (nccl_settle)
  ncclComm_t comm = nullptr;
  ncclResult_t r = ncclCommInitRankConfig(&comm, world, id, rank, &cfg);
  if (r != ncclSuccess && r != ncclInProgress) {
    if (comm) ncclCommAbort(comm);
    return fail(ctx, OCCU_ENCCL, std::string("ncclCommInitRankConfig: ") + ncclGetErrorString(r));
  }
  ctx->comm = comm;
  ctx->comm_aborted = false;
  ctx->rank = rank;
  ctx->world = world;
  return nccl_settle(ctx, "ncclCommInitRankConfig");
}

occu_status occu_dist_set_timeout(occu_ctx *ctx, double seconds) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  if (!(seconds >= 0.0)) return fail(ctx, OCCU_EINVAL, "timeout must be >= 0");
  ctx->nccl_timeout_s = seconds;
  return OCCU_OK;
}

occu_status occu_dist_abort(occu_ctx *ctx) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  if (!ctx->comm) return OCCU_OK;
  nccl_abort(ctx, "aborted by occu_dist_abort");
  return OCCU_OK;
}

occu_status occu_dist_sync(occu_ctx *ctx) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  return stream_wait(ctx, "occu_dist_sync");
}

occu_status occu_save_state(const occu_ctx *cctx, const char *path) {
  occu_ctx *ctx = const_cast<occu_ctx *>(cctx);
  if (!ctx || !path) return fail(ctx, OCCU_EINVAL, "NULL argument");
  const size_t n = ctx->layout.total;
  std::vector<float> m(n), v(n);
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(cudaMemcpyAsync(m.data(), ctx->adam_m.ptr, n * 4, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
  CK(cudaMemcpyAsync(v.data(), ctx->adam_v.ptr, n * 4, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  const int64_t t = ctx->adam_t;
  std::string err;
  if (!write_file(path, "OCCUS001", ctx->cfg, {{&t, 8}, {m.data(), n * 4}, {v.data(), n * 4}}, err))
    return fail(ctx, OCCU_EINVAL, err);
  return OCCU_OK;
}

occu_status occu_load_state(occu_ctx *ctx, const char *path) {
  if (!ctx || !path) return fail(ctx, OCCU_EINVAL, "NULL argument");
  const size_t n = ctx->layout.total;
  std::vector<unsigned char> payload;
  std::string err;
  occu_status st = read_file(path, "OCCUS001", ctx->cfg, payload, 8 + 2 * n * 4, err);
  if (st != OCCU_OK) return fail(ctx, st, "occu_load_state: " + err);
  int64_t t;
  memcpy(&t, payload.data(), 8);
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(cudaMemcpyAsync(ctx->adam_m.ptr, payload.data() + 8, n * 4, cudaMemcpyHostToDevice, ctx->stream), "H2D");
  CK(cudaMemcpyAsync(ctx->adam_v.ptr, payload.data() + 8 + n * 4, n * 4, cudaMemcpyHostToDevice, ctx->stream), "H2D");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  ctx->adam_t = t;
  return OCCU_OK;
}

occu_status occu_set_small_batch_kernel(occu_ctx *ctx, int enable) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  ctx->small_enabled = enable != 0;
  return OCCU_OK;
}

occu_status occu_set_kernel_path(occu_ctx *ctx, int path) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  if (path < 0 || path > 2)
    return fail(ctx, OCCU_EINVAL, "path must be 0 (tensor cores), 1 (SIMT) or 2 (tensor cores, fused aggregation)");
  if (ctx->cfg.prec == OCCU_BF16 && path != 0)
    return fail(ctx, OCCU_EINVAL, "OCCU_BF16 runs on kernel path 0 only");
  if (ctx->cfg.msg == OCCU_MSG_NEIGHBOR_SOFTMAX && path != 0)
    return fail(ctx, OCCU_EINVAL, "reading B (NEIGHBOR_SOFTMAX) runs on kernel path 0 only");
  if (ctx->cfg.readout == OCCU_READOUT_SET_DECODER && path != 0)
    return fail(ctx, OCCU_EINVAL, "the decoder readout runs on kernel path 0 only");
  if (ctx->cfg.graphormer > 0 && path != 0)
    return fail(ctx, OCCU_EINVAL, "Graphormer layers run on kernel path 0 only");
  ctx->path = path;
  return OCCU_OK;
}

occu_status occu_set_keep_intermediates(occu_ctx *ctx, int keep) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  ctx->keep = keep != 0;
  return OCCU_OK;
}

occu_status occu_get_tensor(occu_ctx *ctx, int32_t which, int32_t layer, void *host_dst, size_t bytes) {
  if (!ctx || !host_dst) return fail(ctx, OCCU_EINVAL, "NULL argument");
  if (!ctx->have_forward) return fail(ctx, OCCU_ENOTREADY, "no forward has run");
  const DevCsr &c = ctx->last_csr;
  const int d = ctx->cfg.d;
  const bool per_layer = which <= OCCU_T_H;
  if (per_layer && (layer < 0 || layer >= ctx->cfg.L)) return fail(ctx, OCCU_EINVAL, "bad layer");
  if (per_layer && ctx->small_fwd)
    return fail(ctx, OCCU_ENOTREADY, "the last forward ran the single-CTA small-batch kernel (no per-layer tensors; set keep_intermediates)");
  if (which == OCCU_T_GPH && (layer < 0 || layer >= ctx->cfg.graphormer))
    return fail(ctx, OCCU_EINVAL, "bad Graphormer layer");
  const void *src = nullptr;
  size_t need = 0;
  Workspace &w = ctx->ws;
  switch (which) {
    case OCCU_T_HBAR: src = w.hbar[layer].ptr; need = size_t(c.N) * d * 4; break;
    case OCCU_T_P: src = w.p[layer].ptr; need = size_t(c.N) * 4; break;
    case OCCU_T_Q: src = w.q[layer].ptr; need = size_t(c.N) * 4; break;
    case OCCU_T_E:
      if (layer == ctx->cfg.L - 1 && !ctx->keep)
        return fail(ctx, OCCU_ENOTREADY, "last-layer e not stored (set keep_intermediates)");
      src = w.e[layer].ptr; need = size_t(c.E) * d * 4; break;
    case OCCU_T_H:
      if (layer == ctx->cfg.L - 1 && !ctx->h_last_stored)
        return fail(ctx, OCCU_ENOTREADY, "last-layer h not stored (set keep_intermediates)");
      src = w.h[layer].ptr; need = size_t(c.N) * d * 4; break;
    case OCCU_T_R: src = w.r.ptr; need = size_t(c.B) * ctx->layout.head_in * 4; break;   // [B][d] or [B][k·d]
    case OCCU_T_YHAT: src = w.yhat.ptr; need = size_t(c.B) * 4; break;
    case OCCU_T_GPH: src = w.gh[layer].ptr; need = size_t(c.N) * d * 4; break;
    default: return fail(ctx, OCCU_EINVAL, "unknown tensor");
  }
  if (bytes != need) return fail(ctx, OCCU_EINVAL, "byte count mismatch");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  const bool widen = ctx->cfg.prec == OCCU_BF16 &&
                     (which == OCCU_T_HBAR || which == OCCU_T_E || which == OCCU_T_H);
  if (widen) {     // BF16 stores: copy the 16-bit words, widen to float32 (exact)
    std::vector<uint16_t> tmp(need / 4);
    CK(cudaMemcpyAsync(tmp.data(), src, need / 2, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
    CK(cudaStreamSynchronize(ctx->stream), "sync");
    uint32_t *o = static_cast<uint32_t *>(host_dst);
    for (size_t i = 0; i < tmp.size(); ++i) o[i] = uint32_t(tmp[i]) << 16;
    return OCCU_OK;
  }
  CK(cudaMemcpyAsync(host_dst, src, need, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
  CK(cudaStreamSynchronize(ctx->stream), "sync");
  return OCCU_OK;
}

int64_t occu_last_launch_count(const occu_ctx *ctx) { return ctx ? ctx->launches : 0; }

occu_status occu_set_profiling(occu_ctx *ctx, int enable) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  ctx->prof.on = enable != 0;
  return OCCU_OK;
}

occu_status occu_profile_reset(occu_ctx *ctx) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  cudaSetDevice(ctx->device);
  ctx->prof.reset();
  return OCCU_OK;
}

occu_status occu_profile_query(occu_ctx *ctx, int32_t idx, const char **name, double *total_ms,
                               int64_t *launches) {
  if (!ctx) return fail(nullptr, OCCU_EINVAL, "ctx is NULL");
  cudaSetDevice(ctx->device);
  ctx->prof.drain();
  if (idx < 0 || size_t(idx) >= ctx->prof.names.size()) return fail(ctx, OCCU_EINVAL, "index out of range");
  if (name) *name = ctx->prof.names[idx].c_str();
  if (total_ms) *total_ms = ctx->prof.total_ms[idx];
  if (launches) *launches = ctx->prof.count[idx];
  return OCCU_OK;
}

const char *occu_last_error(const occu_ctx *ctx) {
  if (ctx) return ctx->err.c_str();
  return global_error();
}

}  // extern "C"
