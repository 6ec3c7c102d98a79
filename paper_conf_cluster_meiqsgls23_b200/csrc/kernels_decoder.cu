// NEXT-2 readout: the Set-Transformer decoder of P159-P205 (R30-R34),
//   Decoder(H) = FFN(SAB(PMA_k(H))),  PMA_k(H) = MAB(S, FFN(H)),  SAB(X) = MAB(X, X),
//   MAB(X, Y) = LN(H̄ + FFN(H̄)),  H̄ = LN(X + MHA(X, Y, Y)),
// per graph over its last-layer node states, then the MLP head on the flattened k·d output.
//
// B200 mapping:
//  * FFN(H) over all N nodes is the only large contraction: two tensor-core row-GEMMs with a
//    bias (+ReLU) epilogue (launch_bias_tc), T = ReLU(h W1ᵀ + b1), Z = T W2ᵀ + b2.
//  * MHA(S, Z, Z) needs no per-node key / value projections: the score of node n for seed j
//    in head h is (Q_j,h · (W_k Z_n + b_k)_h)/√d_h = Z_n · M[:, (j,h)] + c_(j,h) with
//    M = W_k,hᵀ Q_j,h / √d_h (d x k·heads, built per CTA from the seeds), and since the
//    attention weights of a (j,h) sum to 1, Σ_n α (W_v Z_n + b_v) = W_v (Σ_n α Z_n) + b_v.  So
//    the pool streams Z once per graph (32-row chunks staged in shared memory) with an online
//    softmax per (j,h), accumulating P_(j,h) = Σ_n α Z_n; W_v is applied to the k·heads pooled
//    vectors only.  Fixed order everywhere (deterministic).
//  * The rest (W_v, W_o, LayerNorms, the k-element SAB, the FFNs, the head) is k-vector work
//    per graph: warp-per-output-row GEMVs against L2-resident weights, one CTA per graph.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdlib.h>
#include <stdint.h>

#include "occu_internal.h"

namespace occu {
namespace {

constexpr int DT = 256;          // threads per CTA
constexpr int NW = DT / 32;
constexpr int CH = 32;           // node rows per pooling chunk
constexpr int KMAX = 8;          // seeds
constexpr int KHMAX = 16;        // seeds x heads
constexpr float L2E = 1.4426950408889634f;

struct DecArgs {
  const float *Z;                // [N][D] FFN(h_L)
  const int32_t *node_off;       // [B+1]
  const float *P;                // flat parameters
  DecLayout L;
  size_t W_1, b_1, w_2, b_2;
  int k, heads, d_h, B;
  float slope;
  float *r, *c, *yhat;           // [B][k·D], [B][d_h], [B]
};

__device__ __forceinline__ float ex2(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// Y[v·ldy + n] = act(bias[n] + Σ_c W[n·ldw + c] X[v·ldx + c]) for rows n < nrows, vectors
// v < nvec; warp per row (strided), lanes stride the columns (coalesced row reads), fixed
// butterfly reduction.  ncols % 4 == 0.
// Rows are taken RB at a time per warp with all RB row loads issued before use (one L2
// latency per batch instead of one per row).
__device__ void warp_gemv(const float *__restrict__ W, int ldw, int ncols, int nrows,
                          const float *X, int ldx, int nvec, float *Y, int ldy,
                          const float *__restrict__ bias, bool relu) {
  constexpr int RB = 8;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  for (int n0 = warp * RB; n0 < nrows; n0 += nw * RB) {
    for (int c0 = 0; c0 < ncols; c0 += 128) {
      const int c = c0 + lane * 4;
      float4 w[RB];
#pragma unroll
      for (int q = 0; q < RB; ++q) {
        const int n = min(n0 + q, nrows - 1);
        w[q] = c < ncols ? __ldg(reinterpret_cast<const float4 *>(W + long(n) * ldw + c))
                         : make_float4(0.f, 0.f, 0.f, 0.f);
      }
      for (int v = 0; v < nvec; ++v) {
        float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
        if (c < ncols) x = *reinterpret_cast<const float4 *>(X + v * ldx + c);
#pragma unroll
        for (int q = 0; q < RB; ++q) {
          float a = w[q].x * x.x + w[q].y * x.y + w[q].z * x.z + w[q].w * x.w;
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
          if (lane == 0 && n0 + q < nrows) {
            float *y = Y + v * ldy + n0 + q;
            *y = (c0 == 0 ? 0.f : *y) + a;
          }
        }
      }
    }
    __syncwarp();
    if (lane < RB && n0 + lane < nrows)
      for (int v = 0; v < nvec; ++v) {
        float *y = Y + v * ldy + n0 + lane;
        const float a = *y + (bias ? __ldg(bias + n0 + lane) : 0.f);
        *y = relu ? fmaxf(a, 0.f) : a;
      }
    __syncwarp();
  }
}

// Butterfly GEMV for the decoder tail (ncols <= 128, nvec <= 8): Y[v·ldy + n] = act(bias[n] +
// Σ_c W[n·ldw + c] X[v·ldx + c]).  A warp takes RB = 32 / NV rows at once (NV = nvec rounded up
// to a power of two, the padding vectors are zero); lane = 4 columns; the 32 (row, vector)
// partial dots are reduced across the warp by a butterfly reduce-scatter (31 shuffles instead of
// 32 x 5), after which lane l holds output l = q·NV + v.  Fixed order (deterministic).
template <int NV>
__device__ void warp_gemv_bf(const float *__restrict__ W, int ldw, int ncols, int nrows,
                             const float *X, int ldx, int nvec, float *Y, int ldy,
                             const float *__restrict__ bias, bool relu) {
  constexpr int RB = 32 / NV;
  const int nw = blockDim.x >> 5, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int c = lane * 4;
  float4 x[NV];
#pragma unroll
  for (int v = 0; v < NV; ++v)
    x[v] = (v < nvec && c < ncols) ? *reinterpret_cast<const float4 *>(X + v * ldx + c)
                                   : make_float4(0.f, 0.f, 0.f, 0.f);
  for (int n0 = warp * RB; n0 < nrows; n0 += nw * RB) {
    float val[32];
#pragma unroll
    for (int q = 0; q < RB; ++q) {
      const int n = min(n0 + q, nrows - 1);
      const float4 w = c < ncols ? __ldg(reinterpret_cast<const float4 *>(W + long(n) * ldw + c))
                                 : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int v = 0; v < NV; ++v)
        val[q * NV + v] = fmaf(w.x, x[v].x, fmaf(w.y, x[v].y, fmaf(w.z, x[v].z, w.w * x[v].w)));
    }
#pragma unroll
    for (int half = 16; half >= 1; half >>= 1) {
      const bool up = (lane & half) != 0;
#pragma unroll
      for (int i = 0; i < half; ++i) {
        const float send = up ? val[i] : val[i + half];
        const float keep = up ? val[i + half] : val[i];
        val[i] = keep + __shfl_xor_sync(0xffffffffu, send, half);
      }
    }
    const int q = lane / NV, v = lane % NV, n = n0 + q;
    if (v < nvec && n < nrows) {
      const float a = val[0] + (bias ? bias[n] : 0.f);      // bias: global or shared
      Y[v * ldy + n] = relu ? fmaxf(a, 0.f) : a;
    }
  }
}

// dispatch on the vector count (k seeds per graph, <= 8)
__device__ __forceinline__ void gemv_k(const float *__restrict__ W, int ldw, int ncols, int nrows,
                                       const float *X, int ldx, int nvec, float *Y, int ldy,
                                       const float *__restrict__ bias, bool relu) {
  if (nvec <= 1) warp_gemv_bf<1>(W, ldw, ncols, nrows, X, ldx, nvec, Y, ldy, bias, relu);
  else if (nvec <= 2) warp_gemv_bf<2>(W, ldw, ncols, nrows, X, ldx, nvec, Y, ldy, bias, relu);
  else if (nvec <= 4) warp_gemv_bf<4>(W, ldw, ncols, nrows, X, ldx, nvec, Y, ldy, bias, relu);
  else warp_gemv_bf<8>(W, ldw, ncols, nrows, X, ldx, nvec, Y, ldy, bias, relu);
}

// Y[v] = LN(A[v] + Bv[v]) · g + b over D channels (eps 1e-5, biased variance); warp per vector.
template <int D>
__device__ void warp_add_ln(const float *A, const float *Bv, float *Y, int nvec,
                            const float *__restrict__ g, const float *__restrict__ b) {
  constexpr int V = D / 32;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  for (int v = warp; v < nvec; v += nw) {
    float x[V], s = 0.f;
#pragma unroll
    for (int i = 0; i < V; ++i) {
      x[i] = A[v * D + lane + 32 * i] + Bv[v * D + lane + 32 * i];
      s += x[i];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float mu = s / float(D);
    float q = 0.f;
#pragma unroll
    for (int i = 0; i < V; ++i) q = fmaf(x[i] - mu, x[i] - mu, q);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    const float inv = rsqrtf(q / float(D) + 1e-5f);
#pragma unroll
    for (int i = 0; i < V; ++i) {
      const int ch = lane + 32 * i;
      Y[v * D + ch] = (x[i] - mu) * inv * g[ch] + b[ch];   // g, b: global or shared
    }
  }
}

// Once per forward (one CTA): PMA queries Q = S W_qᵀ + b_q, the folded key map
// M[c][(j,h)] = Σ_i Q[j][h·dh+i] W_k[h·dh+i][c] / √dh and c_(j,h) = Q_j,h · b_k,h / √dh.
template <int D>
__global__ void __launch_bounds__(DT) set_decoder_prep_kernel(const DecArgs a, float *__restrict__ prep) {
  __shared__ __align__(16) float S[KMAX * D], Q[KMAX * D];
  const int k = a.k, heads = a.heads, KH = k * heads, dh = D / heads, t = threadIdx.x;
  const float *P = a.P;
  const DecLayout &L = a.L;
  pdl_trigger();
  pdl_wait();
  for (int i = t; i < k * D; i += DT) S[i] = P[L.S + i];
  __syncthreads();
  warp_gemv(P + L.M1.Wq, D, D, D, S, D, k, Q, D, P + L.M1.bq, false);
  __syncthreads();
  const float isq = rsqrtf(float(dh));
  for (int o = t; o < D * KH; o += DT) {
    const int c = o % D, kh = o / D, j = kh / heads, h = kh % heads;
    float m0 = 0.f, m1 = 0.f, m2 = 0.f, m3 = 0.f;
    for (int i = 0; i < dh; i += 4) {
      m0 = fmaf(Q[j * D + h * dh + i], __ldg(P + L.M1.Wk + long(h * dh + i) * D + c), m0);
      m1 = fmaf(Q[j * D + h * dh + i + 1], __ldg(P + L.M1.Wk + long(h * dh + i + 1) * D + c), m1);
      m2 = fmaf(Q[j * D + h * dh + i + 2], __ldg(P + L.M1.Wk + long(h * dh + i + 2) * D + c), m2);
      m3 = fmaf(Q[j * D + h * dh + i + 3], __ldg(P + L.M1.Wk + long(h * dh + i + 3) * D + c), m3);
    }
    prep[c * KHMAX + kh] = ((m0 + m1) + (m2 + m3)) * isq;
  }
  if (t < KH) {
    const int j = t / heads, h = t % heads;
    float m = 0.f;
    for (int i = 0; i < dh; ++i) m = fmaf(Q[j * D + h * dh + i], __ldg(P + L.M1.bk + h * dh + i), m);
    prep[D * KHMAX + t] = m * isq;
  }
}

// Pool (PMA's attention of the k seeds over the graph's nodes), split over SPLIT contiguous
// node ranges per graph: CTA (g, s) writes its unnormalised online-softmax state
// (running max m, sum l, Σ 2^{(score - m)·log2e} Z) per (seed, head) to part.
constexpr int SPLIT = 8;
template <int D>
constexpr int part_stride() { return KHMAX * D + 2 * KHMAX; }

template <int D>
__global__ void __launch_bounds__(DT) set_decoder_pool_kernel(const DecArgs a, const float *__restrict__ prep,
                                                              float *__restrict__ part) {
  extern __shared__ __align__(16) float sm[];
  const int k = a.k, heads = a.heads, KH = k * heads;
  float *Zc = sm;                          // [CH][D]
  float *sc = Zc + CH * D;                 // [CH][KHMAX]  scores, then weights
  float *Msm = sc + CH * KHMAX;            // [CH][NW][KHMAX] score partials
  float *Pacc = Msm + CH * NW * KHMAX;     // [KHMAX][D]
  float *cst = Pacc + KHMAX * D;           // [KHMAX]
  float *mrun = cst + KHMAX, *lrun = mrun + KHMAX, *scl = lrun + KHMAX;
  const int t = threadIdx.x;
  const int g = blockIdx.x, sp = blockIdx.y;
  pdl_trigger();
  pdl_wait();
  const long g0 = a.node_off[g], len = a.node_off[g + 1] - g0;
  const long u0 = g0 + len * sp / SPLIT, u1 = g0 + len * (sp + 1) / SPLIT;

  // ---- the folded key map M, c of the seeds' queries (set_decoder_prep_kernel, R32);
  // thread t keeps M[cg·CPG .. +CPG][t & 15] in registers for the score dots
  constexpr int CPG = D / 16;              // channels per group (16 groups of the 256 threads)
  const int cg = t >> 4;
  float mreg[CPG];
#pragma unroll
  for (int i = 0; i < CPG; ++i) mreg[i] = __ldg(prep + (cg * CPG + i) * KHMAX + (t & 15));
  float *red = Msm;                        // [CH][NW][KHMAX] score partials (M lives in registers)
  if (t < KH) {
    cst[t] = prep[D * KHMAX + t];
    mrun[t] = -INFINITY;
    lrun[t] = 0.f;
  }
  for (int i = t; i < KH * D; i += DT) Pacc[i] = 0.f;
  __syncthreads();

  // ---- attention pool over the graph's nodes: online softmax per (seed, head)
  for (long n0 = u0; n0 < u1; n0 += CH) {
    const int rows = int(min(long(CH), u1 - n0));
    for (int i = t; i < rows * (D / 4); i += DT) {
      const int r = i / (D / 4), c4 = i % (D / 4);
      reinterpret_cast<float4 *>(Zc + r * D)[c4] =
          __ldg(reinterpret_cast<const float4 *>(a.Z + (n0 + r) * D) + c4);
    }
    __syncthreads();
    {   // scores: thread (kh, channel group) holds its M slice in registers; partial dots of
        // the two channel groups of a warp combined by shuffle, the NW warp partials in smem
      for (int r = 0; r < rows; ++r) {
        const float *zr = Zc + r * D + cg * CPG;
        float part = 0.f;
#pragma unroll
        for (int i = 0; i < CPG; i += 4) {
          const float4 z = *reinterpret_cast<const float4 *>(zr + i);
          part = fmaf(z.x, mreg[i], fmaf(z.y, mreg[i + 1], fmaf(z.z, mreg[i + 2], fmaf(z.w, mreg[i + 3], part))));
        }
        part += __shfl_xor_sync(0xffffffffu, part, 16);
        if ((t & 16) == 0) red[(r * NW + (t >> 5)) * KHMAX + (t & 15)] = part;
      }
      __syncthreads();
      for (int o = t; o < rows * KH; o += DT) {
        const int r = o / KH, kh = o % KH;
        float sacc = cst[kh];
        for (int w = 0; w < NW; ++w) sacc += red[(r * NW + w) * KHMAX + kh];
        sc[r * KHMAX + kh] = sacc;
      }
    }
    __syncthreads();
    {   // warp per (seed, head): lanes = chunk rows; max, weights and their sum by shuffles
      const int warp = t >> 5, lane = t & 31;
      for (int kh = warp; kh < KH; kh += NW) {
        const float sv = lane < rows ? sc[lane * KHMAX + kh] : -INFINITY;
        float cm = sv;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) cm = fmaxf(cm, __shfl_xor_sync(0xffffffffu, cm, o));
        const float mold = mrun[kh];
        const float mn = fmaxf(mold, cm);
        const float w = lane < rows ? ex2((sv - mn) * L2E) : 0.f;
        float ws = w;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
        if (lane < rows) sc[lane * KHMAX + kh] = w;
        __syncwarp();
        if (lane == 0) {
          const float f = ex2((mold - mn) * L2E);               // 0 on the first chunk
          scl[kh] = f;
          lrun[kh] = lrun[kh] * f + ws;
          mrun[kh] = mn;
        }
      }
    }
    __syncthreads();
    for (int o4 = t; o4 < KH * D / 4; o4 += DT) {   // 4 consecutive channels of one (j,h)
      const int kh = o4 / (D / 4), c = (o4 % (D / 4)) * 4;
      float4 acc = reinterpret_cast<float4 *>(Pacc)[o4];
      const float f = scl[kh];
      acc.x *= f; acc.y *= f; acc.z *= f; acc.w *= f;
      for (int r = 0; r < rows; ++r) {
        const float w = sc[r * KHMAX + kh];
        const float4 z = *reinterpret_cast<const float4 *>(Zc + r * D + c);
        acc.x = fmaf(w, z.x, acc.x); acc.y = fmaf(w, z.y, acc.y);
        acc.z = fmaf(w, z.z, acc.z); acc.w = fmaf(w, z.w, acc.w);
      }
      reinterpret_cast<float4 *>(Pacc)[o4] = acc;
    }
    __syncthreads();
  }
  float *out = part + (long(g) * SPLIT + sp) * part_stride<D>();
  for (int o = t; o < KH * D; o += DT) out[o] = Pacc[o];
  if (t < KH) {
    out[KHMAX * D + t] = mrun[t];
    out[KHMAX * D + KHMAX + t] = lrun[t];
  }
}

// Pool on the legacy tensor path (mma.sync m16n8k16, fp16x2 3-product split = FP32 accuracy):
// per 32-row chunk of Z, the scores S[32][16] = Z·M (4 warps, one 16x8 tile each, K = D) and
// the weighted sums P[16][D] += W[16][32]·Z[32][D] (8 warps, D/64 n-tile pairs each); the
// online softmax bookkeeping (per (seed, head) column over the chunk's rows) stays on CUDA cores.
__device__ __forceinline__ void dsplit_h2(float x0, float x1, uint32_t &hi, uint32_t &lo) {
  const __half2 h = __floats2half2_rn(x0, x1);
  const float2 hf = __half22float2(h);
  const __half2 l = __floats2half2_rn(x0 - hf.x, x1 - hf.y);
  hi = *reinterpret_cast<const uint32_t *>(&h);
  lo = *reinterpret_cast<const uint32_t *>(&l);
}
__device__ __forceinline__ void dmma(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ void dldsm4(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}
__device__ __forceinline__ void dldsm4t(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}
__device__ __forceinline__ void dldsm2(uint32_t addr, uint32_t &r0, uint32_t &r1) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0,%1}, [%2];" : "=r"(r0), "=r"(r1) : "r"(addr));
}
__device__ __forceinline__ uint32_t dsm(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int D>
struct PoolSmem {
  static constexpr int ZS = D + 8;         // halves per Z row (16-byte rows, ldmatrix conflict-free)
  static constexpr int WS = CH + 8;        // halves per W row
  __half zh[CH * ZS], zl[CH * ZS];
  __half mh[KHMAX * ZS], ml[KHMAX * ZS];   // Mᵀ [kh][c]
  __half wh[KHMAX * WS], wl[KHMAX * WS];   // softmax weights [kh][row]
  float sc[CH][KHMAX + 1];
  float cst[KHMAX], mrun[KHMAX], lrun[KHMAX], scl[KHMAX];
};

template <int D>
__global__ void __launch_bounds__(DT) set_decoder_pool_mma_kernel(const DecArgs a, const float *__restrict__ prep,
                                                                  float *__restrict__ part) {
  extern __shared__ __align__(16) unsigned char pool_raw[];
  PoolSmem<D> &S = *reinterpret_cast<PoolSmem<D> *>(pool_raw);
  constexpr int ZS = PoolSmem<D>::ZS, WS = PoolSmem<D>::WS;
  constexpr int NTP = D >= 128 ? D / 128 : 1;   // n-tile pairs of P per warp (D = 128: 8 warps x 16 columns)
  const int KH = a.k * a.heads;
  const int t = threadIdx.x, warp = t >> 5, lane = t & 31, g = lane >> 2, tq = lane & 3;
  const int gi = blockIdx.x, sp = blockIdx.y;
  pdl_trigger();
  pdl_wait();
  const long g0 = a.node_off[gi], len = a.node_off[gi + 1] - g0;
  const long u0 = g0 + len * sp / SPLIT, u1 = g0 + len * (sp + 1) / SPLIT;
  // Mᵀ (columns kh >= KH zero) and the offsets
  for (int i = t; i < KHMAX * D; i += DT) {
    const int kh = i / D, c = i % D;
    const float v = kh < KH ? __ldg(prep + c * KHMAX + kh) : 0.f;
    const __half h = __float2half_rn(v);
    S.mh[kh * ZS + c] = h;
    S.ml[kh * ZS + c] = __float2half_rn(v - __half2float(h));
  }
  if (t < KHMAX) {
    S.cst[t] = t < KH ? prep[D * KHMAX + t] : 0.f;
    S.mrun[t] = -INFINITY;
    S.lrun[t] = 0.f;
  }
  // P accumulators: warp owns n-tiles [warp·2·NTP/2 ...]: for D = 128, n-tiles 2w, 2w + 1
  float pacc[2 * NTP][4];
#pragma unroll
  for (int n = 0; n < 2 * NTP; ++n) pacc[n][0] = pacc[n][1] = pacc[n][2] = pacc[n][3] = 0.f;
  const int nbase = warp * 2 * NTP;        // first n-tile of this warp (8-column tiles)
  const bool pw = nbase * 8 < D;           // warps beyond D/8/(2·NTP) idle in the P product
  __syncthreads();
  for (long n0 = u0; n0 < u1; n0 += CH) {
    const int rows = int(min(long(CH), u1 - n0));
    // ---- Z chunk -> fp16 hi / lo (rows past the range zero)
    for (int i = t; i < CH * (D / 4); i += DT) {
      const int r = i / (D / 4), c = (i % (D / 4)) * 4;
      float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
      if (r < rows) z = __ldg(reinterpret_cast<const float4 *>(a.Z + (n0 + r) * D + c));
      uint32_t h0, l0, h1, l1;
      dsplit_h2(z.x, z.y, h0, l0);
      dsplit_h2(z.z, z.w, h1, l1);
      *reinterpret_cast<uint2 *>(&S.zh[r * ZS + c]) = make_uint2(h0, h1);
      *reinterpret_cast<uint2 *>(&S.zl[r * ZS + c]) = make_uint2(l0, l1);
    }
    __syncthreads();
    // ---- scores: warp w < 4 -> rows (w >> 1)·16.., seeds·heads (w & 1)·8..
    if (warp < 4) {
      const int mt = warp >> 1, nt = warp & 1;
      float c4[4] = {0.f, 0.f, 0.f, 0.f};
      const int arow = mt * 16 + (lane & 7) + ((lane >> 3) & 1) * 8, acol = (lane >> 4) * 8;
      const int brow = nt * 8 + (lane & 7), bcol = ((lane >> 3) & 1) * 8;
#pragma unroll
      for (int ks = 0; ks < D / 16; ++ks) {
        uint32_t ah[4], al[4], bh0, bh1, bl0, bl1;
        dldsm4(dsm(&S.zh[arow * ZS + ks * 16 + acol]), ah);
        dldsm4(dsm(&S.zl[arow * ZS + ks * 16 + acol]), al);
        dldsm2(dsm(&S.mh[brow * ZS + ks * 16 + bcol]), bh0, bh1);
        dldsm2(dsm(&S.ml[brow * ZS + ks * 16 + bcol]), bl0, bl1);
        dmma(c4, al, bh0, bh1);
        dmma(c4, ah, bl0, bl1);
        dmma(c4, ah, bh0, bh1);
      }
      const int r0 = mt * 16 + g, col = nt * 8 + 2 * tq;
      S.sc[r0][col] = r0 < rows ? c4[0] + S.cst[col] : -INFINITY;
      S.sc[r0][col + 1] = r0 < rows ? c4[1] + S.cst[col + 1] : -INFINITY;
      S.sc[r0 + 8][col] = r0 + 8 < rows ? c4[2] + S.cst[col] : -INFINITY;
      S.sc[r0 + 8][col + 1] = r0 + 8 < rows ? c4[3] + S.cst[col + 1] : -INFINITY;
    }
    __syncthreads();
    // ---- online softmax per (seed, head) column over the chunk's rows: warp per column
    for (int kh = warp; kh < KHMAX; kh += NW) {
      const float sv = S.sc[lane][kh];
      float cm = sv;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) cm = fmaxf(cm, __shfl_xor_sync(0xffffffffu, cm, o));
      const float mold = S.mrun[kh];
      const float mn = fmaxf(mold, cm);
      const float ref = mn == -INFINITY ? 0.f : mn;
      const float w = kh < KH ? ex2((sv - ref) * L2E) : 0.f;      // rows past the range: 0
      float ws = w;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
      const __half wh = __float2half_rn(w);
      S.wh[kh * WS + lane] = wh;
      S.wl[kh * WS + lane] = __float2half_rn(w - __half2float(wh));
      __syncwarp();                          // every lane has read mrun[kh] / lrun[kh]
      if (lane == 0) {
        const float f = ex2((mold - ref) * L2E);                   // 0 on the first chunk
        S.scl[kh] = f;
        S.lrun[kh] = S.lrun[kh] * f + ws;
        S.mrun[kh] = mn;
      }
    }
    __syncthreads();
    // ---- P[16][D] = P · scl + W[16][32] · Z[32][D]
    if (pw) {
      const float fa = S.scl[g], fb = S.scl[g + 8];
#pragma unroll
      for (int n = 0; n < 2 * NTP; ++n) {
        pacc[n][0] *= fa; pacc[n][1] *= fa; pacc[n][2] *= fb; pacc[n][3] *= fb;
      }
      const int arow = (lane & 7) + ((lane >> 3) & 1) * 8, acol = (lane >> 4) * 8;
#pragma unroll
      for (int ks = 0; ks < CH / 16; ++ks) {
        uint32_t ah[4], al[4];
        dldsm4(dsm(&S.wh[arow * WS + ks * 16 + acol]), ah);
        dldsm4(dsm(&S.wl[arow * WS + ks * 16 + acol]), al);
        const int brow = ks * 16 + (lane & 7) + ((lane >> 3) & 1) * 8;
#pragma unroll
        for (int np = 0; np < NTP; ++np) {
          const int bcol = (nbase + 2 * np + (lane >> 4)) * 8;
          uint32_t bh[4], bl[4];
          dldsm4t(dsm(&S.zh[brow * ZS + bcol]), bh);
          dldsm4t(dsm(&S.zl[brow * ZS + bcol]), bl);
          dmma(pacc[2 * np], al, bh[0], bh[1]);
          dmma(pacc[2 * np], ah, bl[0], bl[1]);
          dmma(pacc[2 * np], ah, bh[0], bh[1]);
          dmma(pacc[2 * np + 1], al, bh[2], bh[3]);
          dmma(pacc[2 * np + 1], ah, bl[2], bl[3]);
          dmma(pacc[2 * np + 1], ah, bh[2], bh[3]);
        }
      }
    }
    __syncthreads();
  }
  float *out = part + (long(gi) * SPLIT + sp) * part_stride<D>();
  if (pw) {
#pragma unroll
    for (int n = 0; n < 2 * NTP; ++n) {
      const int c = (nbase + n) * 8 + 2 * tq;
      if (g < KH) *reinterpret_cast<float2 *>(out + g * D + c) = make_float2(pacc[n][0], pacc[n][1]);
      if (g + 8 < KH) *reinterpret_cast<float2 *>(out + (g + 8) * D + c) = make_float2(pacc[n][2], pacc[n][3]);
    }
  }
  if (t < KH) {
    out[KHMAX * D + t] = S.mrun[t];
    out[KHMAX * D + KHMAX + t] = S.lrun[t];
  }
}

// GPC graphs per CTA: combine each graph's SPLIT pool partials in fixed order, then the
// MAB / SAB / FFN chain and the head as GEMVs over all GPC·k vectors of the CTA (every weight
// row read from L2 once per CTA serves GPC graphs).
constexpr int GPC = 1;
constexpr int DT_TAIL = 256;   // tail CTA: 8 warps (all B CTAs resident at once)
constexpr int NPV = 20;         // the tail's bias / LayerNorm vectors
template <int D>
constexpr size_t tail_smem_floats(int d_h) {
  return size_t(GPC) * (KMAX * KMAX * 8 + KHMAX * D + 6 * KMAX * D + SPLIT * KHMAX + KHMAX + d_h) +
         size_t(NPV) * D + size_t(KMAX) * D;
}

template <int D>
__global__ void __launch_bounds__(DT_TAIL) set_decoder_kernel(const DecArgs a, const float *__restrict__ part) {
  extern __shared__ __align__(16) float sm[];
  const int k = a.k, heads = a.heads, KH = k * heads, dh = D / heads;
  const int g0 = blockIdx.x * GPC;
  const int G = min(GPC, a.B - g0);          // graphs of this CTA
  const int V = G * k;                       // vectors of the CTA ([graph][seed])
  float *Zc = sm;                            // [GPC][heads][k][k] SAB scores
  float *Pacc = Zc + GPC * KMAX * KMAX * 8;  // [GPC][KH][D]
  float *buf = Pacc + GPC * KHMAX * D;       // 6 x [GPC·k][D]
  constexpr int BS = GPC * KMAX * D;
  float *B0 = buf, *B1 = B0 + BS, *B2 = B1 + BS, *B3 = B2 + BS, *B4 = B3 + BS, *B5 = B4 + BS;
  float *fs = B5 + BS;                       // [GPC][SPLIT][KHMAX] partial scale factors
  float *lsum = fs + GPC * SPLIT * KHMAX;    // [GPC][KHMAX]
  float *cvec = lsum + GPC * KHMAX;          // [GPC][d_h]
  float *pv = cvec + GPC * a.d_h;            // [NPV][D] biases / LayerNorm vectors, then S [k][D]
  const int t = threadIdx.x;
  const DecLayout &L = a.L;
  const float isq = rsqrtf(float(dh));
  pdl_trigger();
  pdl_wait();
  {   // every small parameter vector of the chain into shared memory at once (one L2 latency)
    const size_t vo[NPV] = {L.M1.bv, L.M1.bo, L.M1.ln1_g, L.M1.ln1_b, L.M1.F.b1, L.M1.F.b2,
                            L.M1.ln2_g, L.M1.ln2_b, L.M2.bq, L.M2.bk, L.M2.bv, L.M2.bo,
                            L.M2.ln1_g, L.M2.ln1_b, L.M2.F.b1, L.M2.F.b2, L.M2.ln2_g, L.M2.ln2_b,
                            L.D.b1, L.D.b2};
    for (int i = t; i < NPV * D; i += DT_TAIL) pv[i] = __ldg(a.P + vo[i / D] + i % D);
    for (int i = t; i < k * D; i += DT_TAIL) pv[NPV * D + i] = __ldg(a.P + L.S + i);
  }
  const float *P = a.P;
  auto PV = [&](int i) -> const float * { return pv + i * D; };
  constexpr int PS = part_stride<D>();
  for (int o = t; o < G * KH; o += DT_TAIL) {     // global max, factors 2^{(m_s - M)·log2e}, total sum
    const int gg = o / KH, kh = o % KH;
    const float *pg = part + long(g0 + gg) * SPLIT * PS;
    float M = -INFINITY;
    for (int q = 0; q < SPLIT; ++q) M = fmaxf(M, pg[q * PS + KHMAX * D + kh]);
    float l = 0.f;
    for (int q = 0; q < SPLIT; ++q) {
      const float mq = pg[q * PS + KHMAX * D + kh];
      const float f = mq == -INFINITY ? 0.f : ex2((mq - M) * L2E);
      fs[(gg * SPLIT + q) * KHMAX + kh] = f;
      l = fmaf(pg[q * PS + KHMAX * D + KHMAX + kh], f, l);
    }
    lsum[gg * KHMAX + kh] = l;
  }
  __syncthreads();
  for (int o = t; o < G * KH * D; o += DT_TAIL) {
    const int gg = o / (KH * D), r = o % (KH * D), kh = r / D;
    const float *pg = part + long(g0 + gg) * SPLIT * PS;
    float acc = 0.f;
    for (int q = 0; q < SPLIT; ++q) acc = fmaf(pg[q * PS + r], fs[(gg * SPLIT + q) * KHMAX + kh], acc);
    Pacc[o] = acc / lsum[gg * KHMAX + kh];    // [gg][kh][c] = [(gg·k + j)·heads + h][c]
  }
  __syncthreads();

  // ---- MAB1 = PMA_k: O = W_v P + b_v per head, X1 = W_o O + b_o, H̄ = LN(S + X1), LN(H̄ + FFN(H̄))
  for (int h = 0; h < heads; ++h)
    gemv_k(P + L.M1.Wv + long(h) * dh * D, D, D, dh, Pacc + h * D, heads * D, V, B0 + h * dh, D,
              PV(0) + h * dh, false);
  __syncthreads();
  gemv_k(P + L.M1.Wo, D, D, D, B0, D, V, B1, D, PV(1), false);
  for (int i = t; i < V * D; i += DT_TAIL) B3[i] = pv[NPV * D + i % (k * D)];
  __syncthreads();
  warp_add_ln<D>(B3, B1, B2, V, PV(2), PV(3));      // B2 = H̄1
  __syncthreads();
  gemv_k(P + L.M1.F.W1, D, D, D, B2, D, V, B3, D, PV(4), true);
  __syncthreads();
  gemv_k(P + L.M1.F.W2, D, D, D, B3, D, V, B4, D, PV(5), false);
  __syncthreads();
  warp_add_ln<D>(B2, B4, B5, V, PV(6), PV(7));      // B5 = PMA_k(Z)
  __syncthreads();

  // ---- MAB2 = SAB over each graph's k vectors
  gemv_k(P + L.M2.Wq, D, D, D, B5, D, V, B0, D, PV(8), false);
  gemv_k(P + L.M2.Wk, D, D, D, B5, D, V, B1, D, PV(9), false);
  gemv_k(P + L.M2.Wv, D, D, D, B5, D, V, B2, D, PV(10), false);
  __syncthreads();
  const int HKK = heads * k * k;
  for (int o = t; o < G * HKK; o += DT_TAIL) {     // scores per (graph, head, query, key)
    const int gg = o / HKK, r = o % HKK;
    const int h = r / (k * k), j = (r / k) % k, jj = r % k;
    const float *qv = B0 + (gg * k + j) * D + h * dh, *kv = B1 + (gg * k + jj) * D + h * dh;
    float s = 0.f;
    for (int i = 0; i < dh; ++i) s = fmaf(qv[i], kv[i], s);
    Zc[o] = s * isq;
  }
  __syncthreads();
  for (int o = t; o < G * heads * k; o += DT_TAIL) {   // softmax over the k keys
    float m = -INFINITY, l = 0.f;
    for (int jj = 0; jj < k; ++jj) m = fmaxf(m, Zc[o * k + jj]);
    for (int jj = 0; jj < k; ++jj) {
      const float w = ex2((Zc[o * k + jj] - m) * L2E);
      Zc[o * k + jj] = w;
      l += w;
    }
    for (int jj = 0; jj < k; ++jj) Zc[o * k + jj] /= l;
  }
  __syncthreads();
  for (int o = t; o < V * D; o += DT_TAIL) {
    const int v = o / D, gg = v / k, j = v % k, ch = o % D, h = ch / dh;
    const float *w = Zc + gg * HKK + (h * k + j) * k;
    float acc = 0.f;
    for (int jj = 0; jj < k; ++jj) acc = fmaf(w[jj], B2[(gg * k + jj) * D + ch], acc);
    B3[o] = acc;
  }
  __syncthreads();
  gemv_k(P + L.M2.Wo, D, D, D, B3, D, V, B4, D, PV(11), false);
  __syncthreads();
  warp_add_ln<D>(B5, B4, B0, V, PV(12), PV(13));      // B0 = H̄2
  __syncthreads();
  gemv_k(P + L.M2.F.W1, D, D, D, B0, D, V, B1, D, PV(14), true);
  __syncthreads();
  gemv_k(P + L.M2.F.W2, D, D, D, B1, D, V, B2, D, PV(15), false);
  __syncthreads();
  warp_add_ln<D>(B0, B2, B3, V, PV(16), PV(17));      // B3 = SAB(PMA_k(Z))
  __syncthreads();

  // ---- final FFN -> decoder output [k][D] per graph (flattened into r), then the head
  gemv_k(P + L.D.W1, D, D, D, B3, D, V, B4, D, PV(18), true);
  __syncthreads();
  gemv_k(P + L.D.W2, D, D, D, B4, D, V, B5, D, PV(19), false);
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) a.r[long(g0) * k * D + i] = B5[i];
  warp_gemv(P + a.W_1, k * D, k * D, a.d_h, B5, k * D, G, cvec, a.d_h, P + a.b_1, false);
  __syncthreads();
  const int warp = t >> 5, lane = t & 31;
  if (warp < G) {      // ŷ = w_2 · LReLU(c) + b_2, fixed-order warp reduction, warp per graph
    const int g = g0 + warp;
    float s = 0.f;
    for (int i = lane; i < a.d_h; i += 32) {
      const float cv = cvec[warp * a.d_h + i];
      a.c[long(g) * a.d_h + i] = cv;
      s = fmaf(__ldg(P + a.w_2 + i), cv > 0.f ? cv : a.slope * cv, s);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) a.yhat[g] = s + __ldg(P + a.b_2);
  }
}

}  // namespace

int launch_set_decoder(const occu_ctx *ctx, const DevCsr &csr, const float *hL, float *T, float *Z,
                       float *r, float *c, float *yhat, cudaStream_t st) {
  const occu_config &cf = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  const float *P = ctx->params.as<float>();
  if (!L.dec || cf.k > KMAX || cf.k * cf.heads > KHMAX) return -int(cudaErrorInvalidValue);
  int n = 0, rr;
  if ((rr = launch_bias_tc(ctx, hL, cf.d, csr.N, 0, cf.L, P + L.D.P.b1, true, T, "dec_ffn_tc", st)) < 0) return rr;
  n += rr;
  if ((rr = launch_bias_tc(ctx, T, cf.d, csr.N, 1, cf.L, P + L.D.P.b2, false, Z, "dec_ffn_tc", st)) < 0) return rr;
  n += rr;
  DecArgs a{};
  if (!ctx->ws.dprep.ptr) const_cast<occu_ctx *>(ctx)->dprep_version = -1;   // fresh buffer
  if (const_cast<occu_ctx *>(ctx)->ws.dprep.ensure(size_t(cf.d * KHMAX + KHMAX) * 4) != cudaSuccess)
    return -int(cudaErrorMemoryAllocation);
  float *prep = ctx->ws.dprep.as<float>();
  a.Z = Z; a.node_off = csr.node_off; a.P = P; a.L = L.D;
  a.W_1 = L.W_1; a.b_1 = L.b_1; a.w_2 = L.w_2; a.b_2 = L.b_2;
  a.k = cf.k; a.heads = cf.heads; a.d_h = cf.d_h; a.slope = cf.slope; a.B = csr.B;
  a.r = r; a.c = c; a.yhat = yhat;
  const int D = cf.d;
  if (const_cast<occu_ctx *>(ctx)->ws.dpool.ensure(size_t(csr.B) * SPLIT * (KHMAX * D + 2 * KHMAX) * 4) != cudaSuccess)
    return -int(cudaErrorMemoryAllocation);
  float *part = ctx->ws.dpool.as<float>();
  const size_t smem_pool = size_t(CH * D + CH * KHMAX + CH * NW * KHMAX + KHMAX * D + 4 * KHMAX) * 4;
  const size_t smem_tail = (D == 64 ? tail_smem_floats<64>(cf.d_h) : tail_smem_floats<128>(cf.d_h)) * 4;
  const dim3 gpool(csr.B, SPLIT);
  int nprep = 0;
  static const bool simt_pool = [] {
    const char *e = getenv("OCCU_DEC_POOL_SIMT");
    return e && atoi(e) != 0;
  }();
  const size_t smem_mma = D == 64 ? sizeof(PoolSmem<64>) : sizeof(PoolSmem<128>);
  auto run = [&](auto prepk, auto poolk, auto poolm, auto tailk) {
    if (ctx->dprep_version != ctx->params_version) {   // parameters changed: rebuild M, c
      OCCU_PROF_BEGIN(ctx, "set_decoder_prep", st);
      prepk<<<1, DT, 0, st>>>(a, prep);
      OCCU_PROF_END(ctx);
      const_cast<occu_ctx *>(ctx)->dprep_version = ctx->params_version;
      ++nprep;
    }
    OCCU_PROF_BEGIN(ctx, "set_decoder_pool", st);
    if (simt_pool) {
      cudaFuncSetAttribute(poolk, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem_pool));
      launch_pdl(ctx->pdl & 8, poolk, gpool, DT, smem_pool, st, a, (const float *)prep, part);
    } else {
      cudaFuncSetAttribute(poolm, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem_mma));
      launch_pdl(ctx->pdl & 8, poolm, gpool, DT, smem_mma, st, a, (const float *)prep, part);
    }
    OCCU_PROF_END(ctx);
    OCCU_PROF_BEGIN(ctx, "set_decoder", st);
    cudaFuncSetAttribute(tailk, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem_tail));
    launch_pdl(ctx->pdl & 8, tailk, (csr.B + GPC - 1) / GPC, DT_TAIL, smem_tail, st, a, (const float *)part);
    OCCU_PROF_END(ctx);
  };
  if (D == 64)
    run(set_decoder_prep_kernel<64>, set_decoder_pool_kernel<64>, set_decoder_pool_mma_kernel<64>,
        set_decoder_kernel<64>);
  else
    run(set_decoder_prep_kernel<128>, set_decoder_pool_kernel<128>, set_decoder_pool_mma_kernel<128>,
        set_decoder_kernel<128>);
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? n + 2 + nprep : -int(e);
}

}  // namespace occu
