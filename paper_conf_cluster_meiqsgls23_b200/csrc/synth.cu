// NEXT-4: on-device feature synthesis (R39).  A DL-model family's
// training DAG has one topology for all hyperparameter variants (P237), so a batch of variants
// is built on the GPU from per-family templates (uploaded once) plus four numbers per graph:
//  * the batch CSR is the templates' own CSR (packed once by occu_pack) replicated with the
//    graph offsets — bit-identical to occu_pack of the concatenated graphs, because packing
//    sorts inside each graph and offsets preserve the keys' order;
//  * every hyperparameter-dependent Table I quantity (P97-P123, P129-P133) is a polynomial of
//    degree <= 1 in batch, <= 1 in cin, <= 2 in seq, stored in tensor-product Newton form
//    (occu_gen/templates.py) and evaluated here in float64 (exact for the integer quantities),
//    then encoded log2(1 + x) / 40 like the generator.
// Per step only B x (template, batch, cin, seq, hw) crosses PCIe instead of ~350 B per node.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "occu_internal.h"

struct occu_template {
  int32_t n, m;
  int32_t max_in_degree;
  int device;
  void *dmem;               // one device allocation holding everything below
  const int32_t *in_ptr, *in_src, *in_dst, *in_eid, *out_ptr, *out_pos;
  const float *nstatic, *estatic;   // [n][80], [m][4]
  const uint32_t *code;             // [n·22 + m] sparse polynomial codes: (start << 12) | mask
  const double *coef;               // packed non-zero Newton coefficients
};

namespace occu {
namespace {

constexpr int NQ = 22, NC = 12, FN = 80, FE = 4;
constexpr double BN0 = 4.0, CN0 = 1.0, SN0 = 16.0, SN1 = 32.0;   // Newton nodes (templates.py)

struct SynthGraph {       // per graph of the batch (uploaded per call)
  const int32_t *in_ptr, *in_src, *in_dst, *in_eid, *out_ptr, *out_pos;
  const float *nstatic, *estatic;
  const uint32_t *code;     // sparse polynomials: node quantities [n][22], then edges [m]
  const double *coef;
  int32_t n, m, node_off, edge_off;
  float hp[4];            // batch, cin, seq, hw
};

// log2(1 + 0) / 40 = 0 exactly: the many zero quantities (unused operator-hp slots) skip the log
__device__ __forceinline__ float enc(double x) { return x == 0.0 ? 0.f : float(log2(1.0 + x) / 40.0); }

__device__ __forceinline__ void newton_basis(const float *hp, double (&bv)[NC]) {
  const double nb[2] = {1.0, double(hp[0]) - BN0};
  const double nc[2] = {1.0, double(hp[1]) - CN0};
  const double s = double(hp[2]);
  const double ns[3] = {1.0, s - SN0, (s - SN0) * (s - SN1)};
#pragma unroll
  for (int i = 0; i < 2; ++i)
#pragma unroll
    for (int j = 0; j < 2; ++j)
#pragma unroll
      for (int k = 0; k < 3; ++k) bv[i * 6 + j * 3 + k] = nb[i] * nc[j] * ns[k];
}

// Sparse Newton form: bit mi of the code's low 12 bits marks a non-zero coefficient mi; the
// non-zeros are packed from index code >> 12 on.  Summed in coefficient order — the skipped
// terms are exact zeros, so the result equals the dense sum.
__device__ __forceinline__ double poly(uint32_t code, const double *__restrict__ c, const double (&bv)[NC]) {
  double q = 0.0;
  uint32_t idx = code >> 12;
#pragma unroll
  for (int mi = 0; mi < NC; ++mi)
    if (code & (1u << mi)) q += __ldg(c + idx++) * bv[mi];
  return q;
}

// CTA (graph b, slice s): nodes [64 s, 64 s + 64) and edges [128 s, 128 s + 128) of graph b
// (slices past the graph's end exit at once).  Phase 1: CSR replication with the graph's
// offsets and the 22 node quantities + edge bytes (Newton form, float64) encoded into shared
// memory; phase 2: the 64 node rows [64][80] written coalesced from the template's static
// columns and the encoded values.
constexpr int SN = 64, SE = 128, ST = 256;
__global__ void __launch_bounds__(ST) synth_kernel(const SynthGraph *__restrict__ gs, int B, int N, int E,
                                                   int32_t *node_off, int32_t *edge_off,
                                                   int32_t *in_ptr, int32_t *out_ptr, int32_t *in_src,
                                                   int32_t *in_dst, int32_t *in_eid, int32_t *out_pos,
                                                   int32_t *node_graph, float *__restrict__ nf,
                                                   float *__restrict__ ef) {
  __shared__ float qv[SN][NQ + 5];       // encoded quantities (22), 4 x sizes (4), pad
  __shared__ float cfgv[4];
  const int b = blockIdx.x, sl = blockIdx.y, t = threadIdx.x;
  const SynthGraph &g = gs[b];
  const int n = g.n, m = g.m;
  const int u0 = sl * SN, k0 = sl * SE;
  if (u0 >= n && k0 >= m) return;
  const int n0 = g.node_off, e0 = g.edge_off;
  if (t == 0 && sl == 0) {
    node_off[b] = n0;
    edge_off[b] = e0;
    if (b == B - 1) {
      node_off[B] = N;
      edge_off[B] = E;
      in_ptr[N] = E;
      out_ptr[N] = E;
    }
  }
  double bv[NC];
  newton_basis(g.hp, bv);
  const int un = max(0, min(SN, n - u0)), kn = max(0, min(SE, m - k0));
  if (t < un) {
    const int u = u0 + t;
    in_ptr[n0 + u] = e0 + __ldg(g.in_ptr + u);
    out_ptr[n0 + u] = e0 + __ldg(g.out_ptr + u);
    node_graph[n0 + u] = b;
  }
  if (t < kn) {
    const int k = k0 + t;
    in_src[e0 + k] = n0 + __ldg(g.in_src + k);
    in_dst[e0 + k] = n0 + __ldg(g.in_dst + k);
    in_eid[e0 + k] = e0 + __ldg(g.in_eid + k);
    out_pos[e0 + k] = e0 + __ldg(g.out_pos + k);
    const double x = poly(__ldg(g.code + size_t(n) * NQ + k), g.coef, bv);
    const size_t er = size_t(e0 + k) * FE;
    *reinterpret_cast<float4 *>(ef + er) =
        make_float4(__ldg(g.estatic + size_t(k) * FE), __ldg(g.estatic + size_t(k) * FE + 1), enc(x),
                    __ldg(g.estatic + size_t(k) * FE + 3));
  }
  if (t < 4) cfgv[t] = enc(double(g.hp[t]));
  for (int i = t; i < un * NQ; i += ST) {        // the 22 quantities of the slice's nodes
    const int r = i / NQ, q = i % NQ;
    const double x = poly(__ldg(g.code + size_t(u0 + r) * NQ + q), g.coef, bv);
    qv[r][q] = enc(x);
    if (q >= 16 && q < 20) qv[r][NQ + (q - 16)] = enc(4.0 * x);     // bytes = 4 x size
  }
  __syncthreads();
  for (int i = t; i < un * FN; i += ST) {
    const int r = i / FN, c = i % FN;
    float v;
    if (c >= 42 && c < 58) v = qv[r][c - 42];                  // operator hp
    else if (c >= 58 && c < 62) v = cfgv[c - 58];              // model configuration
    else if (c >= 62 && c < 66) v = 0.f;
    else if (c >= 66 && c < 70) v = qv[r][16 + (c - 66)];      // tensor sizes
    else if (c >= 70 && c < 74) v = qv[r][NQ + (c - 70)];      // bytes
    else if (c == 74 || c == 75) v = qv[r][20 + (c - 74)];     // FLOPs, temp
    else v = __ldg(g.nstatic + size_t(u0) * FN + i);           // hp-independent
    nf[size_t(n0 + u0) * FN + i] = v;
  }
}

occu_status fail(occu_ctx *ctx, occu_status st, const std::string &msg) {
  if (ctx) ctx->err = msg;
  else set_global_error(msg);
  return st;
}
occu_status cuda_fail(occu_ctx *ctx, cudaError_t e, const char *where) {
  return fail(ctx, e == cudaErrorMemoryAllocation ? OCCU_ENOMEM : OCCU_ECUDA,
              std::string(where) + ": " + cudaGetErrorString(e));
}
#define CK(call, where)                                         \
  do {                                                          \
    cudaError_t e__ = (call);                                   \
    if (e__ != cudaSuccess) return cuda_fail(ctx, e__, where);  \
  } while (0)

}  // namespace
}  // namespace occu

using namespace occu;

extern "C" occu_status occu_template_create(occu_ctx *ctx, const occu_graph_view *graph,
                                            const float *node_static, const double *node_coef,
                                            const float *edge_static, const double *edge_coef,
                                            occu_template **out) {
  if (!ctx || !graph || !node_static || !node_coef || !out ||
      (graph->num_edges > 0 && (!edge_static || !edge_coef)))
    return fail(ctx, OCCU_EINVAL, "occu_template_create: NULL argument");
  *out = nullptr;
  occu_csr_batch *h = nullptr;
  occu_status st = occu_pack(graph, 1, &h);      // validates the graph (ids, self-loops)
  if (st != OCCU_OK) return fail(ctx, st, std::string("occu_template_create: ") + global_error());
  const size_t n = size_t(graph->num_nodes), m = size_t(graph->num_edges);
  // sparse polynomial codes: (start << 12) | non-zero mask, node quantities then edges
  std::vector<uint32_t> codes(n * NQ + m);
  std::vector<double> packed;
  for (size_t pi = 0; pi < n * NQ + m; ++pi) {
    const double *c = pi < n * NQ ? node_coef + pi * NC : edge_coef + (pi - n * NQ) * NC;
    uint32_t mask = 0;
    const size_t start = packed.size();
    for (int mi = 0; mi < NC; ++mi)
      if (c[mi] != 0.0) {
        mask |= 1u << mi;
        packed.push_back(c[mi]);
      }
    if (start >= (size_t(1) << 20)) {
      occu_batch_free(h);
      return fail(ctx, OCCU_EINVAL, "occu_template_create: more than 2^20 non-zero coefficients");
    }
    codes[pi] = uint32_t(start << 12) | mask;
  }
  // layout (bytes): ints [in_ptr n+1 | out_ptr n+1 | in_src m | in_dst m | in_eid m | out_pos m |
  // codes n·22+m], then (16-aligned) doubles [packed non-zeros], floats [nstatic n·80 | estatic m·4]
  const size_t ni = 2 * (n + 1) + 4 * m + codes.size();
  const size_t off_d = ((ni * 4 + 15) / 16) * 16;
  const size_t nd = packed.size();
  const size_t off_f = off_d + ((nd * 8 + 15) / 16) * 16;
  const size_t total = off_f + (n * FN + m * FE) * 4;
  std::vector<unsigned char> hbuf(total, 0);
  int32_t *ip = reinterpret_cast<int32_t *>(hbuf.data());
  memcpy(ip, h->in_ptr, (n + 1) * 4);
  memcpy(ip + (n + 1), h->out_ptr, (n + 1) * 4);
  memcpy(ip + 2 * (n + 1), h->in_src, m * 4);
  memcpy(ip + 2 * (n + 1) + m, h->in_dst, m * 4);
  memcpy(ip + 2 * (n + 1) + 2 * m, h->in_eid, m * 4);
  memcpy(ip + 2 * (n + 1) + 3 * m, h->out_pos, m * 4);
  const int32_t tmaxdeg = h->max_in_degree;
  occu_batch_free(h);
  memcpy(ip + 2 * (n + 1) + 4 * m, codes.data(), codes.size() * 4);
  if (nd) memcpy(hbuf.data() + off_d, packed.data(), nd * 8);
  memcpy(hbuf.data() + off_f, node_static, n * FN * 4);
  if (m) memcpy(hbuf.data() + off_f + n * FN * 4, edge_static, m * FE * 4);
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  void *d = nullptr;
  CK(cudaMalloc(&d, total), "template alloc");
  cudaError_t e = cudaMemcpy(d, hbuf.data(), total, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) {
    cudaFree(d);
    return cuda_fail(ctx, e, "template H2D");
  }
  occu_template *t = new occu_template;
  t->n = int32_t(n);
  t->max_in_degree = tmaxdeg;
  t->m = int32_t(m);
  t->device = ctx->device;
  t->dmem = d;
  const int32_t *di = static_cast<const int32_t *>(d);
  t->in_ptr = di;
  t->out_ptr = di + (n + 1);
  t->in_src = di + 2 * (n + 1);
  t->in_dst = t->in_src + m;
  t->in_eid = t->in_dst + m;
  t->out_pos = t->in_eid + m;
  const unsigned char *db = static_cast<const unsigned char *>(d);
  t->code = reinterpret_cast<const uint32_t *>(t->out_pos + m);
  t->coef = reinterpret_cast<const double *>(db + off_d);
  t->nstatic = reinterpret_cast<const float *>(db + off_f);
  t->estatic = t->nstatic + n * FN;
  *out = t;
  return OCCU_OK;
}

extern "C" void occu_template_destroy(occu_template *t) {
  if (!t) return;
  cudaFree(t->dmem);
  delete t;
}

extern "C" occu_status occu_synthesize(occu_ctx *ctx, const occu_template *const *templates,
                                       int32_t num_graphs, const float *hp,
                                       occu_csr_batch **csr_out, float **node_feat,
                                       float **edge_feat) {
  if (!ctx || !templates || !hp || !csr_out || !node_feat || !edge_feat || num_graphs < 1)
    return fail(ctx, OCCU_EINVAL, "occu_synthesize: NULL argument or num_graphs < 1");
  if (ctx->cfg.F_n != FN || ctx->cfg.F_e != FE)
    return fail(ctx, OCCU_EINVAL, "occu_synthesize: the templates carry Table I rows (F_n = 80, F_e = 4)");
  std::vector<SynthGraph> gs(num_graphs);
  int64_t N = 0, E = 0;
  int slices = 1;
  int32_t maxdeg = 0;
  for (int b = 0; b < num_graphs; ++b) {
    const occu_template *t = templates[b];
    if (!t) return fail(ctx, OCCU_EINVAL, "occu_synthesize: NULL template");
    if (t->device != ctx->device) return fail(ctx, OCCU_EINVAL, "occu_synthesize: template on another device");
    for (int j = 0; j < 4; ++j)
      if (!(hp[4 * b + j] >= 0.f) || !isfinite(hp[4 * b + j]))
        return fail(ctx, OCCU_EINVAL, "occu_synthesize: hyperparameters must be finite and >= 0");
    SynthGraph &g = gs[b];
    g.in_ptr = t->in_ptr; g.in_src = t->in_src; g.in_dst = t->in_dst; g.in_eid = t->in_eid;
    g.out_ptr = t->out_ptr; g.out_pos = t->out_pos;
    g.nstatic = t->nstatic; g.estatic = t->estatic; g.code = t->code; g.coef = t->coef;
    g.n = t->n; g.m = t->m;
    g.node_off = int32_t(N);
    g.edge_off = int32_t(E);
    memcpy(g.hp, hp + 4 * b, 16);
    N += t->n;
    E += t->m;
    slices = std::max(slices, std::max((t->n + SN - 1) / SN, (t->m + SE - 1) / SE));
    maxdeg = std::max(maxdeg, t->max_in_degree);
    if (N >= INT32_MAX || E >= INT32_MAX) return fail(ctx, OCCU_EINVAL, "occu_synthesize: N or E >= 2^31");
  }
  Workspace &w = ctx->ws;
  const size_t B1 = size_t(num_graphs) + 1, N1 = size_t(N) + 1;
  const size_t ints = 2 * B1 + 2 * N1 + 4 * size_t(E) + size_t(N);
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(w.scsr.ensure(ints * 4), "synth csr alloc");
  CK(w.snf.ensure(std::max<size_t>(size_t(N) * FN * 4, 4)), "synth node_feat alloc");
  CK(w.sef.ensure(std::max<size_t>(size_t(E) * FE * 4, 4)), "synth edge_feat alloc");
  CK(w.sdesc.ensure(gs.size() * sizeof(SynthGraph)), "synth desc alloc");
  // pageable H2D: staged before cudaMemcpyAsync returns, so the host vector may go away
  CK(cudaMemcpyAsync(w.sdesc.ptr, gs.data(), gs.size() * sizeof(SynthGraph), cudaMemcpyHostToDevice,
                     ctx->stream), "synth desc H2D");
  int32_t *q = w.scsr.as<int32_t>();
  occu_csr_batch *c = static_cast<occu_csr_batch *>(calloc(1, sizeof(occu_csr_batch)));
  if (!c) return fail(ctx, OCCU_ENOMEM, "occu_synthesize: host alloc");
  c->num_graphs = num_graphs;
  c->num_nodes = int32_t(N);
  c->num_edges = int32_t(E);
  c->node_off = q; q += B1;
  c->edge_off = q; q += B1;
  c->in_ptr = q; q += N1;
  c->out_ptr = q; q += N1;
  c->in_src = q; q += E;
  c->in_dst = q; q += E;
  c->in_eid = q; q += E;
  c->out_pos = q; q += E;
  c->node_graph = q;
  c->on_device = 1;
  c->max_in_degree = maxdeg;
  c->priv = nullptr;          // arrays are ctx-owned (valid until the next occu_synthesize)
  OCCU_PROF_BEGIN(ctx, "synthesize", ctx->stream);
  synth_kernel<<<dim3(num_graphs, slices), ST, 0, ctx->stream>>>(
      w.sdesc.as<SynthGraph>(), num_graphs, int(N), int(E), c->node_off, c->edge_off, c->in_ptr,
      c->out_ptr, c->in_src, c->in_dst, c->in_eid, c->out_pos, c->node_graph, w.snf.as<float>(),
      w.sef.as<float>());
  OCCU_PROF_END(ctx);
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    free(c);
    return cuda_fail(ctx, e, "synthesize");
  }
  ++ctx->launches;
  *csr_out = c;
  *node_feat = w.snf.as<float>();
  *edge_feat = w.sef.as<float>();
  return OCCU_OK;
}
