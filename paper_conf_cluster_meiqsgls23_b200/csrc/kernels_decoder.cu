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

// =========================================================================================
// Training through the decoder readout (NEXT-2; oracle.set_decoder_bwd, R46).
//
// Per graph g (CTA per graph, dec_tail_bwd_kernel): the tail is recomputed from the pool
// partials exactly as set_decoder_kernel forms it, every k-row intermediate kept in shared
// memory, then the chain is differentiated backwards from dr = ∂L/∂(decoder output):
//   FFN_D, SAB (= MAB2: LN2, FFN, LN1, W_o, the k x k attention per head, W_q/W_k/W_v),
//   PMA's tail (MAB1: LN2, FFN, LN1, W_o)  ->  dO1 = ∂L/∂(W_v P̄ + b_v) per (seed, head).
// Weight gradients need sums over graphs: each graph writes its (input, output-gradient) rows
// to row arrays [B·k][d] and the backward's fixed-order split-K wgrad kernels, column sums and
// LayerNorm parameter sums form them afterwards.  The node side (dec_pool_bwd_kernel) uses
// the folded key map of the forward: score s_n = Z_n·M_kh + c_kh, α = softmax_n(s), so with
// u_kh = W_v,hᵀ dO1_kh:  ∂α_n = Z_n·u_kh,  ds_n = α_n (∂α_n − Σ_m α_m ∂α_m),
//   ∂Z_n = Σ_kh (α_n,kh u_kh + ds_n,kh M_kh),   G_kh = Σ_n ds_n,kh Z_n,  σ_kh = Σ_n ds_n,kh,
// and the seeds' query gradient ∂q_kh = (W_k,h G_kh + b_k,h σ_kh)/√d_h, where σ_kh = 0 exactly
// (so ∂b_k = 0); ∂α and G are formed relative to the graph's first node (dec_pool_bwd_kernel),
// ∂W_k,h = Σ_j (q_jh/√d_h) ⊗ G_jh summed over graphs (dec_seed_grads_kernel).
// =========================================================================================

// Row-array slots written by dec_tail_bwd_kernel ([B·k][D] each).
enum DecRow {
  R_UD, R_dUD, R_sab, R_dsab, R_T4, R_U2, R_dU2, R_Hb2, R_dT4, R_dHb2, R_T3, R_O2, R_dT3,
  R_dQ2, R_dK2, R_dV2, R_pma, R_dpma, R_T2, R_U1, R_dU1, R_Hb1, R_dT2, R_dHb1, R_T1, R_O1,
  R_dT1, R_dO1, R_COUNT
};

// Y[v][c] (+)= Σ_n X[v][n] W[n·ldw + c] for c < ncols, n < nrows, v < nvec (transposed GEMV):
// warps split the rows n, lane = 4 columns (coalesced W rows), warp partials summed in warp
// order through shared memory (scratch [NW][nvec][ncols]).  Fixed order.
__device__ void gemv_t(const float *__restrict__ W, int ldw, int nrows, int ncols, const float *X, int ldx,
                       int nvec, float *Y, int ldy, float *scratch, bool acc) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  const int per = (nrows + nw - 1) / nw, nb = warp * per, ne = min(nrows, nb + per);
  for (int c0 = 0; c0 < ncols; c0 += 128) {
    const int c = c0 + lane * 4;
    float4 a[KMAX];
#pragma unroll
    for (int v = 0; v < KMAX; ++v) a[v] = make_float4(0.f, 0.f, 0.f, 0.f);
    if (c < ncols)
      for (int n = nb; n < ne; ++n) {
        const float4 w = __ldg(reinterpret_cast<const float4 *>(W + long(n) * ldw + c));
#pragma unroll
        for (int v = 0; v < KMAX; ++v)
          if (v < nvec) {
            const float x = X[v * ldx + n];
            a[v].x = fmaf(x, w.x, a[v].x); a[v].y = fmaf(x, w.y, a[v].y);
            a[v].z = fmaf(x, w.z, a[v].z); a[v].w = fmaf(x, w.w, a[v].w);
          }
      }
    if (c < ncols)
#pragma unroll
      for (int v = 0; v < KMAX; ++v)
        if (v < nvec) *reinterpret_cast<float4 *>(scratch + (warp * KMAX + v) * 128 + lane * 4) = a[v];
    __syncthreads();
    for (int o = threadIdx.x; o < nvec * 128; o += blockDim.x) {
      const int v = o / 128, cc = o % 128;
      if (c0 + cc < ncols) {
        float t = 0.f;
        for (int w2 = 0; w2 < nw; ++w2) t += scratch[(w2 * KMAX + v) * 128 + cc];
        float *y = Y + v * ldy + c0 + cc;
        *y = acc ? *y + t : t;
      }
    }
    __syncthreads();
  }
}

// LayerNorm backward per vector (warp per vector): x = the LN input rows, dy = ∂L/∂y;
// dx (=, or += with acc) rstd·(g⊙dy − mean(g⊙dy) − x̂·mean(g⊙dy⊙x̂)).
template <int D>
__device__ void warp_ln_bwd(const float *x, const float *dy, float *dx, int nvec,
                            const float *__restrict__ g, bool acc) {
  constexpr int V = D / 32;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  for (int v = warp; v < nvec; v += nw) {
    float xv[V], s = 0.f;
#pragma unroll
    for (int i = 0; i < V; ++i) {
      xv[i] = x[v * D + lane + 32 * i];
      s += xv[i];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float mu = s / float(D);
    float q = 0.f;
#pragma unroll
    for (int i = 0; i < V; ++i) q = fmaf(xv[i] - mu, xv[i] - mu, q);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    const float rstd = rsqrtf(q / float(D) + 1e-5f);
    float a1 = 0.f, a2 = 0.f, xh[V], gd[V];
#pragma unroll
    for (int i = 0; i < V; ++i) {
      const int ch = lane + 32 * i;
      xh[i] = (xv[i] - mu) * rstd;
      gd[i] = g[ch] * dy[v * D + ch];
      a1 += gd[i];
      a2 = fmaf(gd[i], xh[i], a2);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      a1 += __shfl_xor_sync(0xffffffffu, a1, o);
      a2 += __shfl_xor_sync(0xffffffffu, a2, o);
    }
    a1 /= float(D);
    a2 /= float(D);
#pragma unroll
    for (int i = 0; i < V; ++i) {
      const int ch = lane + 32 * i;
      const float o = rstd * (gd[i] - a1 - xh[i] * a2);
      dx[v * D + ch] = acc ? dx[v * D + ch] + o : o;
    }
  }
}

struct DecBwdArgs {
  DecArgs f;                     // forward arguments (weights, layout, sizes)
  const float *part;             // pool partials of the forward
  const float *dr;               // [B][k·D] ∂L/∂(decoder output)
  float *rows;                   // [R_COUNT][B·k][D]
  float *pstat;                  // [B][KHMAX][2]: merged pool max, sum
  float *pbar;                   // [B·k·heads][D] merged pooled Z (P̄)
  float *u;                      // [B][KHMAX][D]: W_v,hᵀ dO1_kh
  float *dO1h;                   // [heads][B·k][dh]: ∂O1 head-major
};

template <int D>
constexpr size_t tail_bwd_smem_floats() {
  return size_t(NPV) * D + size_t(KMAX) * D + size_t(KHMAX) * D + 2 * KHMAX + SPLIT * KHMAX +
         size_t(KMAX) * KMAX * 8 * 2 + size_t(30) * KMAX * D + size_t(NW) * KMAX * 128;
}

template <int D>
__global__ void __launch_bounds__(DT_TAIL) dec_tail_bwd_kernel(const DecBwdArgs b) {
  extern __shared__ __align__(16) float sm[];
  const DecArgs &a = b.f;
  const int k = a.k, heads = a.heads, KH = k * heads, dh = D / heads;
  const int g = blockIdx.x, t = threadIdx.x;
  const DecLayout &L = a.L;
  const float *P = a.P;
  const float isq = rsqrtf(float(dh));
  float *pv = sm;                                  // [NPV][D]
  float *Ssm = pv + NPV * D;                       // [KMAX][D] seeds
  float *Pacc = Ssm + KMAX * D;                    // [KHMAX][D]
  float *mstat = Pacc + KHMAX * D, *lsum = mstat + KHMAX;
  float *fs = lsum + KHMAX;                        // [SPLIT][KHMAX]
  float *Watt = fs + SPLIT * KHMAX;                // [heads][k][k] (max 8 x 8 x 8)
  float *dWatt = Watt + KMAX * KMAX * 8;
  float *buf = dWatt + KMAX * KMAX * 8;            // 30 x [KMAX][D]
  float *scr = buf + 30 * KMAX * D;                // gemv_t scratch [NW][KMAX][128]
  auto B = [&](int i) { return buf + i * KMAX * D; };
  const size_t vo[NPV] = {L.M1.bv, L.M1.bo, L.M1.ln1_g, L.M1.ln1_b, L.M1.F.b1, L.M1.F.b2,
                          L.M1.ln2_g, L.M1.ln2_b, L.M2.bq, L.M2.bk, L.M2.bv, L.M2.bo,
                          L.M2.ln1_g, L.M2.ln1_b, L.M2.F.b1, L.M2.F.b2, L.M2.ln2_g, L.M2.ln2_b,
                          L.D.b1, L.D.b2};
  for (int i = t; i < NPV * D; i += DT_TAIL) pv[i] = __ldg(P + vo[i / D] + i % D);
  for (int i = t; i < k * D; i += DT_TAIL) Ssm[i] = __ldg(P + L.S + i);
  auto PV = [&](int i) -> const float * { return pv + i * D; };
  constexpr int PS = part_stride<D>();
  const float *pg = b.part + long(g) * SPLIT * PS;
  for (int kh = t; kh < KH; kh += DT_TAIL) {       // merge exactly as set_decoder_kernel
    float M = -INFINITY;
    for (int q = 0; q < SPLIT; ++q) M = fmaxf(M, pg[q * PS + KHMAX * D + kh]);
    float l = 0.f;
    for (int q = 0; q < SPLIT; ++q) {
      const float mq = pg[q * PS + KHMAX * D + kh];
      const float f = mq == -INFINITY ? 0.f : ex2((mq - M) * L2E);
      fs[q * KHMAX + kh] = f;
      l = fmaf(pg[q * PS + KHMAX * D + KHMAX + kh], f, l);
    }
    mstat[kh] = M;
    lsum[kh] = l;
    b.pstat[(long(g) * KHMAX + kh) * 2] = M;
    b.pstat[(long(g) * KHMAX + kh) * 2 + 1] = l;
  }
  __syncthreads();
  for (int o = t; o < KH * D; o += DT_TAIL) {
    const int kh = o / D;
    float acc = 0.f;
    for (int q = 0; q < SPLIT; ++q) acc = fmaf(pg[q * PS + o], fs[q * KHMAX + kh], acc);
    Pacc[o] = acc / lsum[kh];
    // head-major [heads][B·k][D] (row (g, j) of head h), contiguous per head for the W_v gradient
    const int j = kh / heads, h = kh % heads;
    b.pbar[(long(h) * a.B * k + long(g) * k + j) * D + o % D] = Pacc[o];
  }
  __syncthreads();
  // ---- forward recompute (set_decoder_kernel's chain), every intermediate kept
  float *O1 = B(0), *A1 = B(1), *T1 = B(2), *Hb1 = B(3), *U1 = B(4), *F1 = B(5), *T2 = B(6),
        *pma = B(7), *Q2 = B(8), *K2 = B(9), *V2 = B(10), *O2 = B(11), *A2 = B(12), *T3 = B(13),
        *Hb2 = B(14), *U2 = B(15), *F2 = B(16), *T4 = B(17), *sab = B(18), *UD = B(19);
  float *g0 = B(20), *g1 = B(21), *g2 = B(22), *g3 = B(23), *g4 = B(24), *g5 = B(25), *g6 = B(26),
        *g7 = B(27), *g8 = B(28), *g9 = B(29);
  const int V = k;
  for (int h = 0; h < heads; ++h)
    gemv_k(P + L.M1.Wv + long(h) * dh * D, D, D, dh, Pacc + h * D, heads * D, V, O1 + h * dh, D,
           PV(0) + h * dh, false);
  __syncthreads();
  gemv_k(P + L.M1.Wo, D, D, D, O1, D, V, A1, D, PV(1), false);
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) T1[i] = Ssm[i] + A1[i];
  __syncthreads();
  warp_add_ln<D>(Ssm, A1, Hb1, V, PV(2), PV(3));
  __syncthreads();
  gemv_k(P + L.M1.F.W1, D, D, D, Hb1, D, V, U1, D, PV(4), true);
  __syncthreads();
  gemv_k(P + L.M1.F.W2, D, D, D, U1, D, V, F1, D, PV(5), false);
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) T2[i] = Hb1[i] + F1[i];
  warp_add_ln<D>(Hb1, F1, pma, V, PV(6), PV(7));
  __syncthreads();
  gemv_k(P + L.M2.Wq, D, D, D, pma, D, V, Q2, D, PV(8), false);
  gemv_k(P + L.M2.Wk, D, D, D, pma, D, V, K2, D, PV(9), false);
  gemv_k(P + L.M2.Wv, D, D, D, pma, D, V, V2, D, PV(10), false);
  __syncthreads();
  const int KK = k * k;
  for (int o = t; o < heads * KK; o += DT_TAIL) {
    const int h = o / KK, j = (o / k) % k, jj = o % k;
    float sdot = 0.f;
    for (int i = 0; i < dh; ++i) sdot = fmaf(Q2[j * D + h * dh + i], K2[jj * D + h * dh + i], sdot);
    Watt[o] = sdot * isq;
  }
  __syncthreads();
  for (int o = t; o < heads * k; o += DT_TAIL) {
    float m = -INFINITY, l = 0.f;
    for (int jj = 0; jj < k; ++jj) m = fmaxf(m, Watt[o * k + jj]);
    for (int jj = 0; jj < k; ++jj) {
      const float w = ex2((Watt[o * k + jj] - m) * L2E);
      Watt[o * k + jj] = w;
      l += w;
    }
    for (int jj = 0; jj < k; ++jj) Watt[o * k + jj] /= l;
  }
  __syncthreads();
  for (int o = t; o < V * D; o += DT_TAIL) {
    const int j = o / D, ch = o % D, h = ch / dh;
    const float *w = Watt + (h * k + j) * k;
    float acc = 0.f;
    for (int jj = 0; jj < k; ++jj) acc = fmaf(w[jj], V2[jj * D + ch], acc);
    O2[o] = acc;
  }
  __syncthreads();
  gemv_k(P + L.M2.Wo, D, D, D, O2, D, V, A2, D, PV(11), false);
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) T3[i] = pma[i] + A2[i];
  warp_add_ln<D>(pma, A2, Hb2, V, PV(12), PV(13));
  __syncthreads();
  gemv_k(P + L.M2.F.W1, D, D, D, Hb2, D, V, U2, D, PV(14), true);
  __syncthreads();
  gemv_k(P + L.M2.F.W2, D, D, D, U2, D, V, F2, D, PV(15), false);
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) T4[i] = Hb2[i] + F2[i];
  warp_add_ln<D>(Hb2, F2, sab, V, PV(16), PV(17));
  __syncthreads();
  gemv_k(P + L.D.W1, D, D, D, sab, D, V, UD, D, PV(18), true);
  __syncthreads();
  // ---- backward
  const float *dD = b.dr + long(g) * k * D;
  for (int i = t; i < V * D; i += DT_TAIL) g9[i] = dD[i];
  __syncthreads();
  gemv_t(P + L.D.W2, D, D, D, g9, D, V, g0, D, scr, false);        // ∂UD
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) g0[i] = UD[i] > 0.f ? g0[i] : 0.f;
  __syncthreads();
  gemv_t(P + L.D.W1, D, D, D, g0, D, V, g1, D, scr, false);        // ∂sab
  __syncthreads();
  warp_ln_bwd<D>(T4, g1, g2, V, PV(16), false);                    // ∂T4 (= ∂F2)
  __syncthreads();
  gemv_t(P + L.M2.F.W2, D, D, D, g2, D, V, g3, D, scr, false);     // ∂U2
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) g3[i] = U2[i] > 0.f ? g3[i] : 0.f;
  for (int i = t; i < V * D; i += DT_TAIL) g4[i] = g2[i];          // ∂Hb2 = ∂T4 + FFN part
  __syncthreads();
  gemv_t(P + L.M2.F.W1, D, D, D, g3, D, V, g4, D, scr, true);
  __syncthreads();
  warp_ln_bwd<D>(T3, g4, g5, V, PV(12), false);                    // ∂T3 (= ∂A2, residual ∂pma)
  __syncthreads();
  gemv_t(P + L.M2.Wo, D, D, D, g5, D, V, g6, D, scr, false);       // ∂O2
  __syncthreads();
  // attention over the k seeds: ∂w, ∂s, ∂Q2, ∂K2, ∂V2 (g7 = ∂Q2, g8 = ∂K2, A1 reused as ∂V2)
  float *dQ2 = g7, *dK2 = g8, *dV2 = A2;       // A2 no longer needed after the row record below
  for (int o = t; o < heads * KK; o += DT_TAIL) {
    const int h = o / KK, j = (o / k) % k, jj = o % k;
    float sdot = 0.f;
    for (int i = 0; i < dh; ++i) sdot = fmaf(g6[j * D + h * dh + i], V2[jj * D + h * dh + i], sdot);
    dWatt[o] = sdot;
  }
  __syncthreads();
  for (int o = t; o < heads * k; o += DT_TAIL) {     // ∂s = w (∂w − Σ w ∂w), scaled by 1/√d_h
    float dot = 0.f;
    for (int jj = 0; jj < k; ++jj) dot = fmaf(Watt[o * k + jj], dWatt[o * k + jj], dot);
    for (int jj = 0; jj < k; ++jj) dWatt[o * k + jj] = Watt[o * k + jj] * (dWatt[o * k + jj] - dot) * isq;
  }
  __syncthreads();
  // write the row records that need A2's buffer before it becomes ∂V2
  float *rows = b.rows;
  const long RK = long(a.B) * k;
  auto rec = [&](int slot, const float *src) {
    float *dst = rows + (long(slot) * RK + long(g) * k) * D;
    for (int i = t; i < V * D; i += DT_TAIL) dst[i] = src[i];
  };
  __syncthreads();
  for (int o = t; o < V * D; o += DT_TAIL) {
    const int j = o / D, ch = o % D, h = ch / dh;
    float aq = 0.f, ak = 0.f, av = 0.f;
    for (int jj = 0; jj < k; ++jj) {
      aq = fmaf(dWatt[(h * k + j) * k + jj], K2[jj * D + ch], aq);       // ∂Q2[j]
      ak = fmaf(dWatt[(h * k + jj) * k + j], Q2[jj * D + ch], ak);       // ∂K2[j]
      av = fmaf(Watt[(h * k + jj) * k + j], g6[jj * D + ch], av);        // ∂V2[j]
    }
    dQ2[o] = aq;
    dK2[o] = ak;
    dV2[o] = av;
  }
  __syncthreads();
  // ∂pma = ∂T3 (residual) + W_qᵀ ∂Q2 + W_kᵀ ∂K2 + W_vᵀ ∂V2  -> g9
  for (int i = t; i < V * D; i += DT_TAIL) g9[i] = g5[i];
  __syncthreads();
  gemv_t(P + L.M2.Wq, D, D, D, dQ2, D, V, g9, D, scr, true);
  gemv_t(P + L.M2.Wk, D, D, D, dK2, D, V, g9, D, scr, true);
  gemv_t(P + L.M2.Wv, D, D, D, dV2, D, V, g9, D, scr, true);
  __syncthreads();
  // records of the SAB / final FFN part
  rec(R_UD, UD); rec(R_dUD, g0); rec(R_sab, sab); rec(R_dsab, g1); rec(R_T4, T4);
  rec(R_U2, U2); rec(R_dU2, g3); rec(R_Hb2, Hb2); rec(R_dT4, g2); rec(R_dHb2, g4); rec(R_T3, T3);
  rec(R_O2, O2); rec(R_dT3, g5); rec(R_dQ2, dQ2); rec(R_dK2, dK2); rec(R_dV2, dV2); rec(R_pma, pma);
  rec(R_dpma, g9);
  __syncthreads();
  // PMA tail: ∂T2 = LN2ᵀ(∂pma); ∂U1; ∂Hb1 = ∂T2 + W1ᵀ ∂U1; ∂T1 = LN1ᵀ(∂Hb1); ∂O1 = W_oᵀ ∂T1
  warp_ln_bwd<D>(T2, g9, g0, V, PV(6), false);                     // g0 = ∂T2 (= ∂F1)
  __syncthreads();
  gemv_t(P + L.M1.F.W2, D, D, D, g0, D, V, g1, D, scr, false);
  __syncthreads();
  for (int i = t; i < V * D; i += DT_TAIL) {
    g1[i] = U1[i] > 0.f ? g1[i] : 0.f;                             // g1 = ∂U1 (pre-ReLU)
    g2[i] = g0[i];
  }
  __syncthreads();
  gemv_t(P + L.M1.F.W1, D, D, D, g1, D, V, g2, D, scr, true);      // g2 = ∂Hb1
  __syncthreads();
  warp_ln_bwd<D>(T1, g2, g3, V, PV(2), false);                     // g3 = ∂T1 (= ∂A1 = ∂S_g)
  __syncthreads();
  gemv_t(P + L.M1.Wo, D, D, D, g3, D, V, g4, D, scr, false);       // g4 = ∂O1
  __syncthreads();
  rec(R_T2, T2); rec(R_U1, U1); rec(R_dU1, g1); rec(R_Hb1, Hb1); rec(R_dT2, g0); rec(R_dHb1, g2);
  rec(R_T1, T1); rec(R_O1, O1); rec(R_dT1, g3); rec(R_dO1, g4);
  for (int i = t; i < V * D; i += DT_TAIL) {     // ∂O1 head-major [heads][B·k][dh] (W_v gradient)
    const int j = i / D, ch = i % D, h = ch / dh;
    b.dO1h[(long(h) * a.B * k + long(g) * k + j) * dh + ch % dh] = g4[i];
  }
  // u_kh = W_v,hᵀ ∂O1[j, h-slice]  (the node side's ∂P̄_kh)
  for (int o = t; o < KH * D; o += DT_TAIL) {
    const int kh = o / D, c = o % D, j = kh / heads, h = kh % heads;
    float acc = 0.f;
    for (int i = 0; i < dh; ++i) acc = fmaf(g4[j * D + h * dh + i], __ldg(P + L.M1.Wv + long(h * dh + i) * D + c), acc);
    b.u[(long(g) * KHMAX + kh) * D + c] = acc;
  }
}

// Node side of PMA's attention, pass A (mode 0: per-range partial Σ_n α ∂α per (seed, head))
// and pass B (mode 1: ds, ∂Z rows, per-range partial G_kh = Σ ds Z_n and σ_kh = Σ ds).
// Grid (B, SPLIT) as the forward pool; 32-row chunks of Z staged in shared memory.
struct DecPoolBwdArgs {
  const float *Z, *prep, *pstat, *u;
  const int32_t *node_off;
  int k, heads, B;
  float *dsum_part;              // [B][SPLIT][KHMAX]
  float *dZ;                     // [N][D]
  float *gpart;                  // [B][SPLIT][KHMAX][D + 1]
};

// Every node is taken relative to the graph's first node r: ∂α_n − ∂α_r = (Z_n − Z_r)·u and,
// since Σ_n ds_n = 0 exactly, G_kh = Σ_n ds_n (Z_n − Z_r).  Same values, but node states that
// nearly coincide across a graph no longer cancel at the size of Z itself.
template <int D>
__global__ void __launch_bounds__(DT) dec_pool_bwd_kernel(const DecPoolBwdArgs a, int mode) {
  // the folded key map (prep: [c][kh] + the bias row) and the graph's u vectors are staged in
  // shared memory once per CTA (row strides padded to D + 1: conflict-free column walks);
  // every sum keeps its order (the same bits as reading them from global memory)
  __shared__ float Zc[CH][D + 1];
  __shared__ float al[CH][KHMAX], ds[CH][KHMAX];
  __shared__ float Dsum[KHMAX];
  __shared__ float Zr[D];
  __shared__ float Ps[D * KHMAX + KHMAX];      // prep [c][kh], then the bias row [kh]
  __shared__ float PsT[KHMAX][D + 1];           // prep transposed [kh][c]
  __shared__ float Us[KHMAX][D + 1];            // u of graph g [kh][c]
  const int KH = a.k * a.heads, t = threadIdx.x, g = blockIdx.x, sp = blockIdx.y;
  const long g0 = a.node_off[g], len = a.node_off[g + 1] - g0;
  const long u0 = g0 + len * sp / SPLIT, u1 = g0 + len * (sp + 1) / SPLIT;
  for (int c = t; c < D; c += DT) Zr[c] = __ldg(a.Z + g0 * D + c);
  for (int i = t; i < D * KHMAX + KHMAX; i += DT) {
    const float v = a.prep[i];
    Ps[i] = v;
    if (i < D * KHMAX) PsT[i % KHMAX][i / KHMAX] = v;
  }
  for (int i = t; i < KHMAX * D; i += DT) Us[i / D][i % D] = __ldg(a.u + long(g) * KHMAX * D + i);
  if (mode == 1 && t < KH) {
    float s = 0.f;
    for (int q = 0; q < SPLIT; ++q) s += a.dsum_part[(long(g) * SPLIT + q) * KHMAX + t];
    Dsum[t] = s;
  }
  // per-thread accumulators: mode 0: Σ α ∂α for kh = t (t < KH); mode 1: G[kh][c] for
  // outputs o = t, t + DT, ... of KH·D, and σ_kh
  float acc0 = 0.f;
  float gacc[KHMAX * D / DT];
#pragma unroll
  for (int i = 0; i < KHMAX * D / DT; ++i) gacc[i] = 0.f;
  float sacc = 0.f;
  __syncthreads();
  for (long n0 = u0; n0 < u1; n0 += CH) {
    const int rows = int(min(long(CH), u1 - n0));
    for (int i = t; i < CH * D; i += DT) {
      const int r = i / D, c = i % D;
      Zc[r][c] = r < rows ? __ldg(a.Z + (n0 + r) * D + c) : 0.f;
    }
    __syncthreads();
    for (int o = t; o < rows * KH; o += DT) {       // α and ∂α − ∂α_r of (row, kh)
      const int r = o / KH, kh = o % KH;
      float s = Ps[D * KHMAX + kh], da = 0.f;
#pragma unroll 8
      for (int c = 0; c < D; ++c) {
        s = fmaf(Zc[r][c], Ps[c * KHMAX + kh], s);
        da = fmaf(Zc[r][c] - Zr[c], Us[kh][c], da);
      }
      const float M = a.pstat[(long(g) * KHMAX + kh) * 2], l = a.pstat[(long(g) * KHMAX + kh) * 2 + 1];
      const float alpha = ex2((s - M) * L2E) / l;
      al[r][kh] = alpha;
      ds[r][kh] = mode == 0 ? alpha * da : alpha * (da - Dsum[kh]);
    }
    __syncthreads();
    if (mode == 0) {
      if (t < KH)
        for (int r = 0; r < rows; ++r) acc0 += ds[r][t];
    } else {
      for (int o = t; o < rows * D; o += DT) {      // ∂Z rows
        const int r = o / D, c = o % D;
        float z = 0.f;
        for (int kh = 0; kh < KH; ++kh)
          z = fmaf(al[r][kh], Us[kh][c], fmaf(ds[r][kh], PsT[kh][c], z));
        a.dZ[(n0 + r) * D + c] = z;
      }
#pragma unroll
      for (int i = 0; i < KHMAX * D / DT; ++i) {
        const int o = t + i * DT, kh = o / D, c = o % D;
        if (kh < KH)
          for (int r = 0; r < rows; ++r) gacc[i] = fmaf(ds[r][kh], Zc[r][c] - Zr[c], gacc[i]);
      }
      if (t < KH)
        for (int r = 0; r < rows; ++r) sacc += ds[r][t];
    }
    __syncthreads();
  }
  if (mode == 0) {
    if (t < KH) a.dsum_part[(long(g) * SPLIT + sp) * KHMAX + t] = acc0;
  } else {
    float *gp = a.gpart + (long(g) * SPLIT + sp) * KHMAX * (D + 1);
#pragma unroll
    for (int i = 0; i < KHMAX * D / DT; ++i) {
      const int o = t + i * DT, kh = o / D, c = o % D;
      if (kh < KH) gp[kh * (D + 1) + c] = gacc[i];
    }
    if (t < KH) gp[t * (D + 1) + D] = sacc;
  }
}

// Merge of the pool-backward partials over graphs and ranges, thread per output (kh, c):
// Σ_g Σ_q in float64, g ascending then q ascending (the order the seeds' CTA used to walk
// alone); consecutive threads read consecutive columns of each partial row.
__global__ void __launch_bounds__(256) dec_gpart_reduce_kernel(const float *__restrict__ gpart, int B, int KH,
                                                               int W, float *__restrict__ gsum) {
  const int o = blockIdx.x * 256 + threadIdx.x;
  if (o >= KH * W) return;
  const int kh = o / W, c = o % W;
  double acc = 0.0;
  const long stride = long(KHMAX) * W;
  const float *p = gpart + long(kh) * W + c;
  const long n = long(B) * SPLIT;
  long i = 0;
  for (; i + 8 <= n; i += 8) {
    float v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldg(p + (i + u) * stride);
#pragma unroll
    for (int u = 0; u < 8; ++u) acc += double(v[u]);
  }
  for (; i < n; ++i) acc += double(__ldg(p + i * stride));
  gsum[o] = float(acc);
}

// The seeds' side (one CTA): merge the pool-backward partials over graphs and ranges, then
// ∂q_kh, ∂W_k, ∂b_k, ∂Q1 -> ∂W_q, ∂b_q and ∂S = Σ_g ∂T1_g + W_qᵀ ∂Q1.
template <int D>
__global__ void __launch_bounds__(DT) dec_seed_grads_kernel(const DecArgs a, const float *__restrict__ gpart,
                                                            const float *__restrict__ dT1rows, float *__restrict__ G) {
  __shared__ __align__(16) float Gs[KHMAX][D + 1];
  __shared__ __align__(16) float S[KMAX * D], Q[KMAX * D], dQ[KMAX * D];
  const int k = a.k, heads = a.heads, KH = k * heads, dh = D / heads, t = threadIdx.x;
  const DecLayout &L = a.L;
  const float *P = a.P;
  const float isq = rsqrtf(float(dh));
  for (int o = t; o < KH * (D + 1); o += DT) Gs[o / (D + 1)][o % (D + 1)] = gpart[o];   // merged (dec_gpart_reduce_kernel)
  for (int i = t; i < k * D; i += DT) S[i] = P[L.S + i];
  __syncthreads();
  warp_gemv(P + L.M1.Wq, D, D, D, S, D, k, Q, D, P + L.M1.bq, false);
  __syncthreads();
  // ∂q_kh = (W_k,h G_kh + b_k,h σ_kh)/√d_h -> ∂Q1[j][h·dh + i]; ∂W_k, ∂b_k
  for (int o = t; o < k * D; o += DT) {
    const int j = o / D, n = o % D, h = n / dh;
    const int kh = j * heads + h;
    // σ_kh = Σ_n ds_n is exactly 0 (softmax shift invariance; Gs[kh][D] holds its rounding),
    // so ∂q_kh = W_k,h G_kh / √d_h with G_kh taken relative to the reference node
    float acc = 0.f;
    for (int c = 0; c < D; ++c) acc = fmaf(__ldg(P + L.M1.Wk + long(n) * D + c), Gs[kh][c], acc);
    dQ[o] = acc * isq;
  }
  for (int o = t; o < D * D; o += DT) {
    const int n = o / D, c = o % D, h = n / dh;
    float acc = 0.f;
    for (int j = 0; j < k; ++j) acc = fmaf(Q[j * D + n] * isq, Gs[j * heads + h][c], acc);
    G[L.M1.Wk + o] = acc;
  }
  for (int n = t; n < D; n += DT) G[L.M1.bk + n] = 0.f;     // ∂b_k = Σ q σ / √d_h = 0 exactly
  __syncthreads();
  for (int o = t; o < D * D; o += DT) {            // ∂W_q = Σ_j ∂Q1[j] ⊗ S[j]
    const int n = o / D, c = o % D;
    float acc = 0.f;
    for (int j = 0; j < k; ++j) acc = fmaf(dQ[j * D + n], S[j * D + c], acc);
    G[L.M1.Wq + o] = acc;
  }
  for (int n = t; n < D; n += DT) {
    float acc = 0.f;
    for (int j = 0; j < k; ++j) acc += dQ[j * D + n];
    G[L.M1.bq + n] = acc;
  }
  for (int o = t; o < k * D; o += DT) {            // ∂S = Σ_g ∂T1_g + W_qᵀ ∂Q1
    const int j = o / D, c = o % D;
    double acc = 0.0;
    for (int g = 0; g < a.B; ++g) acc += double(dT1rows[(long(g) * k + j) * D + c]);
    float w = 0.f;
    for (int n = 0; n < D; ++n) w = fmaf(dQ[j * D + n], __ldg(P + L.M1.Wq + long(n) * D + c), w);
    G[L.S + o] = float(acc) + w;
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

namespace occu {

int launch_set_decoder_bwd(occu_ctx *ctx, const DevCsr &csr, const float *hL, const float *T,
                           const float *Z, const float *dr, float *dZ, float *dT, float *dhL,
                           cudaStream_t st) {
  const occu_config &cf = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  const float *P = ctx->params.as<float>();
  float *G = ctx->grads.as<float>();
  const int D = cf.d, k = cf.k, KH = k * cf.heads, B = csr.B;
  if (!L.dec || k > KMAX || KH > KHMAX) return -int(cudaErrorInvalidValue);
  const long RK = long(B) * k;
  const size_t f_rows = size_t(R_COUNT) * RK * D, f_pstat = size_t(B) * KHMAX * 2,
               f_pbar = size_t(B) * KH * D, f_u = size_t(B) * KHMAX * D,
               f_ds = size_t(B) * SPLIT * KHMAX, f_gp = (size_t(B) * SPLIT + 1) * KHMAX * (D + 1),
               f_h = size_t(RK) * D, f_x = size_t(RK) * D;
  if (ctx->ws.dbwd.ensure((f_rows + f_pstat + f_pbar + f_u + f_ds + f_gp + f_h + f_x) * 4) != cudaSuccess)
    return -int(cudaErrorMemoryAllocation);
  float *rows = ctx->ws.dbwd.as<float>(), *pstat = rows + f_rows, *pbar = pstat + f_pstat,
        *u = pbar + f_pbar, *dsp = u + f_u, *gp = dsp + f_ds, *dO1h = gp + f_gp, *xscr = dO1h + f_h;
  DecBwdArgs b{};
  DecArgs &a = b.f;
  a.Z = Z; a.node_off = csr.node_off; a.P = P; a.L = L.D;
  a.W_1 = L.W_1; a.b_1 = L.b_1; a.w_2 = L.w_2; a.b_2 = L.b_2;
  a.k = k; a.heads = cf.heads; a.d_h = cf.d_h; a.slope = cf.slope; a.B = B;
  b.part = ctx->ws.dpool.as<float>(); b.dr = dr; b.rows = rows; b.pstat = pstat; b.pbar = pbar; b.u = u;
  b.dO1h = dO1h;
  int n = 0;
  OCCU_PROF_BEGIN(ctx, "dec_tail_bwd", st);
  const size_t smem = (D == 64 ? tail_bwd_smem_floats<64>() : tail_bwd_smem_floats<128>()) * 4;
  if (D == 64) {
    cudaFuncSetAttribute(dec_tail_bwd_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    dec_tail_bwd_kernel<64><<<B, DT_TAIL, smem, st>>>(b);
  } else {
    cudaFuncSetAttribute(dec_tail_bwd_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    dec_tail_bwd_kernel<128><<<B, DT_TAIL, smem, st>>>(b);
  }
  OCCU_PROF_END(ctx);
  ++n;
  DecPoolBwdArgs pa{};
  pa.Z = Z; pa.prep = ctx->ws.dprep.as<float>(); pa.pstat = pstat; pa.u = u; pa.node_off = csr.node_off;
  pa.k = k; pa.heads = cf.heads; pa.B = B; pa.dsum_part = dsp; pa.dZ = dZ; pa.gpart = gp;
  OCCU_PROF_BEGIN(ctx, "dec_pool_bwd", st);
  for (int mode = 0; mode < 2; ++mode) {
    if (D == 64) dec_pool_bwd_kernel<64><<<dim3(B, SPLIT), DT, 0, st>>>(pa, mode);
    else dec_pool_bwd_kernel<128><<<dim3(B, SPLIT), DT, 0, st>>>(pa, mode);
  }
  OCCU_PROF_END(ctx);
  n += 2;
  OCCU_PROF_BEGIN(ctx, "dec_seed_grads", st);
  {
    // merged partials after the B·SPLIT raw ones (f_gp holds one extra [KHMAX][D + 1] slot)
    float *gsum = gp + size_t(B) * SPLIT * KHMAX * (D + 1);
    const int outs = k * cf.heads * (D + 1);
    dec_gpart_reduce_kernel<<<(outs + 255) / 256, 256, 0, st>>>(gp, B, k * cf.heads, D + 1, gsum);
    if (D == 64) dec_seed_grads_kernel<64><<<1, DT, 0, st>>>(a, gsum, rows + size_t(R_dT1) * RK * D, G);
    else dec_seed_grads_kernel<128><<<1, DT, 0, st>>>(a, gsum, rows + size_t(R_dT1) * RK * D, G);
    ++n;
  }
  OCCU_PROF_END(ctx);
  ++n;
  // tail weight / bias / LayerNorm gradients: fixed-order reductions over the B·k rows
  auto row = [&](int slot) { return rows + size_t(slot) * RK * D; };
  // (the split-K wgrad kernels of the backward, parallel column sums and LayerNorm sums)
  int rr;
  auto wg = [&](const float *X, const float *Y, size_t out) {
    if ((rr = launch_wgrad(ctx, X, D, Y, D, RK, G + out, st, false)) >= 0) n += rr;
  };
  auto cs = [&](const float *X, size_t out) {
    if ((rr = launch_colsum_rows(ctx, X, RK, G + out, st)) >= 0) n += rr;
  };
  auto lg = [&](const float *x, size_t gam, const float *dy, size_t g_, size_t b_) {
    if ((rr = launch_ln_param_grads(ctx, x, P + gam, dy, RK, xscr, G + g_, G + b_, st)) >= 0) n += rr;
  };
  const DecLayout &DL = L.D;
  OCCU_PROF_BEGIN(ctx, "dec_tail_wgrads", st);
  wg(dr, row(R_UD), DL.D.W2); cs(dr, DL.D.b2);
  wg(row(R_dUD), row(R_sab), DL.D.W1); cs(row(R_dUD), DL.D.b1);
  lg(row(R_T4), DL.M2.ln2_g, row(R_dsab), DL.M2.ln2_g, DL.M2.ln2_b);
  wg(row(R_dT4), row(R_U2), DL.M2.F.W2); cs(row(R_dT4), DL.M2.F.b2);
  wg(row(R_dU2), row(R_Hb2), DL.M2.F.W1); cs(row(R_dU2), DL.M2.F.b1);
  lg(row(R_T3), DL.M2.ln1_g, row(R_dHb2), DL.M2.ln1_g, DL.M2.ln1_b);
  wg(row(R_dT3), row(R_O2), DL.M2.Wo); cs(row(R_dT3), DL.M2.bo);
  wg(row(R_dQ2), row(R_pma), DL.M2.Wq); cs(row(R_dQ2), DL.M2.bq);
  wg(row(R_dK2), row(R_pma), DL.M2.Wk); cs(row(R_dK2), DL.M2.bk);
  wg(row(R_dV2), row(R_pma), DL.M2.Wv); cs(row(R_dV2), DL.M2.bv);
  lg(row(R_T2), DL.M1.ln2_g, row(R_dpma), DL.M1.ln2_g, DL.M1.ln2_b);
  wg(row(R_dT2), row(R_U1), DL.M1.F.W2); cs(row(R_dT2), DL.M1.F.b2);
  wg(row(R_dU1), row(R_Hb1), DL.M1.F.W1); cs(row(R_dU1), DL.M1.F.b1);
  lg(row(R_T1), DL.M1.ln1_g, row(R_dHb1), DL.M1.ln1_g, DL.M1.ln1_b);
  wg(row(R_dT1), row(R_O1), DL.M1.Wo); cs(row(R_dT1), DL.M1.bo);
  cs(row(R_dO1), DL.M1.bv);
  const int dh = D / cf.heads;
  for (int h = 0; h < cf.heads; ++h)       // ∂W_v rows of head h: Σ_(g,j) ∂O1[g,j][h] ⊗ P̄[g,(j,h)]
    if ((rr = launch_wgrad(ctx, dO1h + size_t(h) * RK * dh, dh, pbar + size_t(h) * RK * D, D, RK,
                           G + DL.M1.Wv + size_t(h) * dh * D, st, false)) >= 0) n += rr;
  OCCU_PROF_END(ctx);
  if (rr < 0) return rr;
  // PMA's pre-pooling FFN over the N node rows (tensor cores): Z = T W2ᵀ + b2, T = ReLU(h W1ᵀ + b1)
  int r;
  (void)row;
  if ((r = launch_plain_masked_tc(ctx, dZ, D, csr.N, 3, cf.L, nullptr, dT, "dec_ffn_bwd_tc", st, T, 0.f)) < 0) return r;
  n += r;
  if ((r = launch_wgrad(ctx, dZ, D, T, D, csr.N, G + DL.P.W2, st, false)) < 0) return r;
  n += r;
  if ((r = launch_colsum_rows(ctx, dZ, csr.N, G + DL.P.b2, st)) < 0) return r;
  n += r;
  if ((r = launch_plain_tc(ctx, dT, D, csr.N, 2, cf.L, nullptr, dhL, "dec_ffn_bwd_tc", st)) < 0) return r;
  n += r;
  if ((r = launch_wgrad(ctx, dT, D, hL, D, csr.N, G + DL.P.W1, st, false)) < 0) return r;
  n += r;
  if ((r = launch_colsum_rows(ctx, dT, csr.N, G + DL.P.b1, st)) < 0) return r;
  n += r;
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? n : -int(e);
}

}  // namespace occu
