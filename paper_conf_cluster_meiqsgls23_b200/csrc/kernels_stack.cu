// Training through the paper's readout stack (P153-P205 with
// Adam, P273): the backward of the Graphormer layers (pre-LN MHA + FFN over each graph's node
// set, R35-R37) and the building blocks the decoder backward shares with them.
//
//   Graphormer layer (forward, kernels_graphormer.cu):  X1 = LN1(H), Q|K|V = X1 W_{q,k,v}ᵀ + b,
//     O = softmax(Q Kᵀ/√d_h) V per graph and head, h̄ = O W_oᵀ + b_o + H, X2 = LN2(h̄),
//     T = ReLU(X2 W1ᵀ + b1), out = T W2ᵀ + b2 + h̄.
//   Backward (this file), with dX = dY·W row-GEMMs on tensor cores against transposed fp16x2
//   weight images (gph_tslot), weight gradients XᵀY on the split-K tensor-core wgrad kernel,
//   bias / LayerNorm parameter gradients as fixed-order column sums (float64 partials):
//     dT = (dout W2) ⊙ [T > 0]; dX2 = dT W1; dh̄ = dout + LN2ᵀ(dX2); dO = dh̄ W_o;
//     attention backward per graph and head (below); dX1 = dQ W_q + dK W_k + dV W_v;
//     dH = dh̄ + LN1ᵀ(dX1).
//   Attention backward (no atomics; tensor cores for d_h in {16, 32}, the FP32 CUDA-core
//   kernels below for d_h = 64 or with OCCU_ATTN_BWD_SIMT=1): stats m_i, l_i of every query row over
//   its own graph's keys and D_i = Σ_j P_ij (dO_i·V_j) (= <dO_i, O_i>, from the recomputed P,
//   taken relative to the dominant key so that saturated softmax rows do not cancel);
//     dQ_i = Σ_j P_ij (dO_i·V_j − D_i) K_j / √d_h        (thread = query row)
//     dV_j = Σ_i P_ij dO_i,  dK_j = Σ_i P_ij (dO_i·V_j − D_i) Q_i / √d_h   (thread = key row)
//   with P_ij = exp(s_ij − m_i)/l_i recomputed, keys / queries of the block's graphs staged
//   through shared memory; sums in ascending index order (deterministic).
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>

#include "occu_internal.h"

namespace occu {
namespace {

constexpr int ST = 256;          // threads per block (row kernels)

#define SK_CHECK()                                  \
  do {                                              \
    cudaError_t e__ = cudaGetLastError();           \
    if (e__ != cudaSuccess) return -int(e__);       \
  } while (0)

int grid_rows(long rows, int rows_per_block, int cap) {
  return int(std::max<long>(1, std::min<long>((rows + rows_per_block - 1) / rows_per_block, cap)));
}

// ---------------------------------------------------------------------------------------
// LayerNorm backward (R33), warp per row, V = D/32 channels per lane (lane-contiguous):
//   x̂ = (x − μ)·rstd,  dx = add + rstd·(g⊙dy − mean(g⊙dy) − x̂·mean(g⊙dy⊙x̂)),
// and per-block partial column sums of dy⊙x̂ (dγ) and dy (dβ) in float64.
template <int D>
__global__ void __launch_bounds__(ST) ln_bwd_kernel(const float *__restrict__ x, const float *__restrict__ gam,
                                                    const float *__restrict__ dy, const float *__restrict__ add,
                                                    float *__restrict__ dx, long R, double *__restrict__ part) {
  constexpr int V = D / 32;
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  double pg[V], pb[V];
  float gv[V];
#pragma unroll
  for (int c = 0; c < V; ++c) {
    pg[c] = pb[c] = 0.0;
    gv[c] = __ldg(gam + lane * V + c);
  }
  const long nw = long(gridDim.x) * (ST / 32);
  for (long r = long(blockIdx.x) * (ST / 32) + wl; r < R; r += nw) {
    float xv[V], dv[V];
#pragma unroll
    for (int c = 0; c < V; ++c) {
      xv[c] = __ldg(x + r * D + lane * V + c);
      dv[c] = __ldg(dy + r * D + lane * V + c);
    }
    float s = 0.f;
#pragma unroll
    for (int c = 0; c < V; ++c) s += xv[c];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float mu = s * (1.f / float(D));
    float q = 0.f;
#pragma unroll
    for (int c = 0; c < V; ++c) q = fmaf(xv[c] - mu, xv[c] - mu, q);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    const float rstd = rsqrtf(q * (1.f / float(D)) + 1e-5f);
    float a1 = 0.f, a2 = 0.f, xh[V], gd[V];
#pragma unroll
    for (int c = 0; c < V; ++c) {
      xh[c] = (xv[c] - mu) * rstd;
      gd[c] = gv[c] * dv[c];
      a1 += gd[c];
      a2 = fmaf(gd[c], xh[c], a2);
      pg[c] = fma(double(dv[c]), double(xh[c]), pg[c]);
      pb[c] += double(dv[c]);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      a1 += __shfl_xor_sync(0xffffffffu, a1, o);
      a2 += __shfl_xor_sync(0xffffffffu, a2, o);
    }
    a1 *= 1.f / float(D);
    a2 *= 1.f / float(D);
#pragma unroll
    for (int c = 0; c < V; ++c) {
      float o = rstd * (gd[c] - a1 - xh[c] * a2);
      if (add) o += __ldg(add + r * D + lane * V + c);
      dx[r * D + lane * V + c] = o;
    }
  }
  __shared__ double red[ST / 32][2 * D];
#pragma unroll
  for (int c = 0; c < V; ++c) {
    red[wl][lane * V + c] = pg[c];
    red[wl][D + lane * V + c] = pb[c];
  }
  __syncthreads();
  for (int o = threadIdx.x; o < 2 * D; o += ST) {
    double t = 0.0;
    for (int w = 0; w < ST / 32; ++w) t += red[w][o];
    part[long(blockIdx.x) * 2 * D + o] = t;
  }
}

// Per-block partial column sums of X [R][D] (bias gradients), float64, warp per row.
template <int D>
__global__ void __launch_bounds__(ST) colsum_kernel(const float *__restrict__ X, long R,
                                                    double *__restrict__ part) {
  constexpr int V = D / 32;
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  double acc[V];
#pragma unroll
  for (int c = 0; c < V; ++c) acc[c] = 0.0;
  const long nw = long(gridDim.x) * (ST / 32);
  for (long r = long(blockIdx.x) * (ST / 32) + wl; r < R; r += nw) {
#pragma unroll
    for (int c = 0; c < V; ++c) acc[c] += double(__ldg(X + r * D + lane * V + c));
  }
  __shared__ double red[ST / 32][D];
#pragma unroll
  for (int c = 0; c < V; ++c) red[wl][lane * V + c] = acc[c];
  __syncthreads();
  for (int o = threadIdx.x; o < D; o += ST) {
    double t = 0.0;
    for (int w = 0; w < ST / 32; ++w) t += red[w][o];
    part[long(blockIdx.x) * D + o] = t;
  }
}

// out[c] = Σ_b part[b][c] in block order (float64), c < C.  out2 (nullable) takes columns
// [C, 2C) of a [nblk][2C] partial array.
__global__ void col_reduce_kernel(const double *__restrict__ part, int nblk, int C, int ld,
                                  float *__restrict__ out, float *__restrict__ out2) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= C) return;
  double a = 0.0, b = 0.0;
  for (int k = 0; k < nblk; ++k) {
    a += part[long(k) * ld + c];
    if (out2) b += part[long(k) * ld + C + c];
  }
  out[c] = float(a);
  if (out2) out2[c] = float(b);
}

// dA = dh ⊙ LReLU'(h) (÷ deg for MEAN) — sign(A) = sign(h) (R7).
__global__ void mask_dA_kernel(const float *__restrict__ dh, const float *__restrict__ h,
                               const int32_t *__restrict__ in_ptr, long N, int D, int mean,
                               float slope, float *__restrict__ dA) {
  const long total = N * D / 4;
  for (long i = blockIdx.x * long(blockDim.x) + threadIdx.x; i < total; i += long(gridDim.x) * blockDim.x) {
    const long u = i / (D / 4);
    const float4 g = __ldg(reinterpret_cast<const float4 *>(dh) + i);
    const float4 x = __ldg(reinterpret_cast<const float4 *>(h) + i);
    float dsc = 1.f;
    if (mean) {
      const int deg = __ldg(in_ptr + u + 1) - __ldg(in_ptr + u);
      dsc = float(deg > 0 ? deg : 1);
    }
    float4 o;
    o.x = g.x * (x.x > 0.f ? 1.f : slope) / dsc;
    o.y = g.y * (x.y > 0.f ? 1.f : slope) / dsc;
    o.z = g.z * (x.z > 0.f ? 1.f : slope) / dsc;
    o.w = g.w * (x.w > 0.f ? 1.f : slope) / dsc;
    reinterpret_cast<float4 *>(dA)[i] = o;
  }
}

// ---------------------------------------------------------------------------------------
// Attention backward (per graph, per head; block-diagonal over the batch).
struct AttnBwdArgs {
  const float *Q, *K, *V, *O, *dO;   // [N][D]
  const int32_t *node_off, *node_graph;
  float *dQ, *dK, *dV;               // [N][D]
  float *stats;                      // [N][heads][4]: m, l, D', dP_ir (see pass 2)
  int N, D, heads;
  float scale;                       // 1 / sqrt(d_h)
};

constexpr int ABT = 128;             // rows per block
constexpr int TK = 32;               // staged rows per tile

// Pass 1 + dQ: thread = query row i of head blockIdx.y.
template <int DH>
__global__ void __launch_bounds__(ABT) attn_bwd_q_kernel(const AttnBwdArgs a) {
  __shared__ float sk[TK][DH], sv[TK][DH];
  const int h = blockIdx.y;
  const long i0 = long(blockIdx.x) * ABT;
  const long i = i0 + threadIdx.x;
  const bool live = i < a.N;
  const long il = min(i0 + ABT, long(a.N)) - 1;
  const int b0 = __ldg(a.node_graph + i0), b1 = __ldg(a.node_graph + il);
  const int ub = __ldg(a.node_off + b0), ue = __ldg(a.node_off + b1 + 1);   // union key range
  int kb = 0, ke = 0;
  float q[DH], go[DH], acc[DH];
  if (live) {
    const int b = __ldg(a.node_graph + i);
    kb = __ldg(a.node_off + b);
    ke = __ldg(a.node_off + b + 1);
#pragma unroll
    for (int c = 0; c < DH; ++c) {
      q[c] = __ldg(a.Q + i * a.D + h * DH + c) * a.scale;
      go[c] = __ldg(a.dO + i * a.D + h * DH + c);
      acc[c] = 0.f;
    }
  }
  // pass 1: row maximum and normaliser over the own graph's keys
  float m = -INFINITY, l = 0.f;
  int ref = kb;                                  // first key attaining the row maximum
  for (int t0 = ub; t0 < ue; t0 += TK) {
    __syncthreads();
    for (int e = threadIdx.x; e < TK * DH; e += ABT) {
      const int rr = e / DH, cc = e % DH;
      sk[rr][cc] = t0 + rr < ue ? __ldg(a.K + long(t0 + rr) * a.D + h * DH + cc) : 0.f;
    }
    __syncthreads();
    if (live) {
      const int jb = max(kb, t0), je = min(ke, t0 + TK);
      for (int j = jb; j < je; ++j) {
        float s = 0.f;
#pragma unroll
        for (int c = 0; c < DH; ++c) s = fmaf(q[c], sk[j - t0][c], s);
        if (s > m) {
          l = l * expf(m - s) + 1.f;
          m = s;
          ref = j;
        } else {
          l += expf(s - m);
        }
      }
    }
  }
  const float inv_l = 1.f / l;
  // pass 2: D_i = Σ_j P_ij dP_ij taken relative to the dominant key r (the first one at the
  // row maximum): D'_i = Σ_j P_ij (dP_ij − dP_ir) and dS_ij = P_ij ((dP_ij − dP_ir) − D'_i).
  // Same value as P ⊙ (dP − D), but when the softmax saturates (P_ir -> 1) the plain form
  // cancels dP_ir − D ≈ (1 − P_ir)·Δ at a rounding error ~ε|dP_ir| while this form keeps
  // ~ε|Δ| (float64 accumulation, the recomputed P).
  float dpr = 0.f, Dp = 0.f;
  if (live) {
#pragma unroll
    for (int c = 0; c < DH; ++c) dpr = fmaf(go[c], __ldg(a.V + long(ref) * a.D + h * DH + c), dpr);
  }
  {
    double dacc = 0.0;
    for (int t0 = ub; t0 < ue; t0 += TK) {
      __syncthreads();
      for (int e = threadIdx.x; e < TK * DH; e += ABT) {
        const int rr = e / DH, cc = e % DH;
        const bool in = t0 + rr < ue;
        sk[rr][cc] = in ? __ldg(a.K + long(t0 + rr) * a.D + h * DH + cc) : 0.f;
        sv[rr][cc] = in ? __ldg(a.V + long(t0 + rr) * a.D + h * DH + cc) : 0.f;
      }
      __syncthreads();
      if (live) {
        const int jb = max(kb, t0), je = min(ke, t0 + TK);
        for (int j = jb; j < je; ++j) {
          float s = 0.f, dp = 0.f;
#pragma unroll
          for (int c = 0; c < DH; ++c) {
            s = fmaf(q[c], sk[j - t0][c], s);
            dp = fmaf(go[c], sv[j - t0][c], dp);
          }
          dacc = fma(double(expf(s - m) * inv_l), double(dp - dpr), dacc);
        }
      }
    }
    Dp = float(dacc);
  }
  // pass 3: dQ
  for (int t0 = ub; t0 < ue; t0 += TK) {
    __syncthreads();
    for (int e = threadIdx.x; e < TK * DH; e += ABT) {
      const int rr = e / DH, cc = e % DH;
      const bool in = t0 + rr < ue;
      sk[rr][cc] = in ? __ldg(a.K + long(t0 + rr) * a.D + h * DH + cc) : 0.f;
      sv[rr][cc] = in ? __ldg(a.V + long(t0 + rr) * a.D + h * DH + cc) : 0.f;
    }
    __syncthreads();
    if (live) {
      const int jb = max(kb, t0), je = min(ke, t0 + TK);
      for (int j = jb; j < je; ++j) {
        float s = 0.f, dp = 0.f;
#pragma unroll
        for (int c = 0; c < DH; ++c) {
          s = fmaf(q[c], sk[j - t0][c], s);
          dp = fmaf(go[c], sv[j - t0][c], dp);
        }
        const float p = expf(s - m) * inv_l;
        const float ds = p * ((dp - dpr) - Dp);
#pragma unroll
        for (int c = 0; c < DH; ++c) acc[c] = fmaf(ds, sk[j - t0][c], acc[c]);
      }
    }
  }
  if (live) {
#pragma unroll
    for (int c = 0; c < DH; ++c) a.dQ[i * a.D + h * DH + c] = acc[c] * a.scale;
    float *stt = a.stats + (i * a.heads + h) * 4;
    stt[0] = m;
    stt[1] = l;
    stt[2] = Dp;
    stt[3] = dpr;
  }
}

// dK, dV: thread = key row j of head blockIdx.y; queries of the block's graphs staged.
template <int DH>
__global__ void __launch_bounds__(ABT) attn_bwd_kv_kernel(const AttnBwdArgs a) {
  __shared__ float sq[TK][DH], sg[TK][DH], ss[TK][4];
  const int h = blockIdx.y;
  const long j0 = long(blockIdx.x) * ABT;
  const long j = j0 + threadIdx.x;
  const bool live = j < a.N;
  const long jl = min(j0 + ABT, long(a.N)) - 1;
  const int b0 = __ldg(a.node_graph + j0), b1 = __ldg(a.node_graph + jl);
  const int ub = __ldg(a.node_off + b0), ue = __ldg(a.node_off + b1 + 1);
  int qb = 0, qe = 0;
  float k[DH], v[DH], dk[DH], dv[DH];
  if (live) {
    const int b = __ldg(a.node_graph + j);
    qb = __ldg(a.node_off + b);
    qe = __ldg(a.node_off + b + 1);
#pragma unroll
    for (int c = 0; c < DH; ++c) {
      k[c] = __ldg(a.K + j * a.D + h * DH + c);
      v[c] = __ldg(a.V + j * a.D + h * DH + c);
      dk[c] = dv[c] = 0.f;
    }
  }
  for (int t0 = ub; t0 < ue; t0 += TK) {
    __syncthreads();
    for (int e = threadIdx.x; e < TK * DH; e += ABT) {
      const int rr = e / DH, cc = e % DH;
      const bool in = t0 + rr < ue;
      sq[rr][cc] = in ? __ldg(a.Q + long(t0 + rr) * a.D + h * DH + cc) * a.scale : 0.f;
      sg[rr][cc] = in ? __ldg(a.dO + long(t0 + rr) * a.D + h * DH + cc) : 0.f;
    }
    for (int e = threadIdx.x; e < TK * 4; e += ABT) {
      const int rr = e / 4, cc = e % 4;
      ss[rr][cc] = t0 + rr < ue ? a.stats[(long(t0 + rr) * a.heads + h) * 4 + cc] : 1.f;
    }
    __syncthreads();
    if (live) {
      const int ib = max(qb, t0), ie = min(qe, t0 + TK);
      for (int i = ib; i < ie; ++i) {
        const int r = i - t0;
        float s = 0.f, dp = 0.f;
#pragma unroll
        for (int c = 0; c < DH; ++c) {
          s = fmaf(sq[r][c], k[c], s);
          dp = fmaf(sg[r][c], v[c], dp);
        }
        const float p = expf(s - ss[r][0]) / ss[r][1];
        const float ds = p * ((dp - ss[r][3]) - ss[r][2]);
#pragma unroll
        for (int c = 0; c < DH; ++c) {
          dv[c] = fmaf(p, sg[r][c], dv[c]);
          dk[c] = fmaf(ds, sq[r][c], dk[c]);      // sq already carries 1/√d_h
        }
      }
    }
  }
  if (live) {
#pragma unroll
    for (int c = 0; c < DH; ++c) {
      a.dK[j * a.D + h * DH + c] = dk[c];
      a.dV[j * a.D + h * DH + c] = dv[c];
    }
  }
}


// ---------------------------------------------------------------------------------------
// Attention backward on tensor cores (d_h in {16, 32}): the same sums as the CUDA-core kernels
// above (stats, D' relative to the dominant key, dQ; then dK, dV), every product on mma.sync
// m16n8k8 TF32 in the 3-product split (x = hi + lo, hi·hi + hi·lo + lo·hi: ~2^-22 relative,
// the FP32 tolerance; TF32 keeps FP32's exponent range, so the small gradient values need
// no scaling).  CTA = 64 rows (4 warps x 16) of one head; the other side's rows stream
// through shared memory in 64-row blocks, pre-split into hi / lo tiles.  The accumulator
// fragment of S / dP (rows g, g+8; columns 2t, 2t+1 of an 8-wide group) becomes the A operand
// of the next product without shuffles by reading its k index t as column 2t and t + 4 as
// column 2t + 1 (the B rows are read in the same order).  Sums over the quad's four threads
// (softmax stats, D') are combined by xor shuffles (commutative: the same bits on every
// thread).  No atomics: dQ on the query side, dK / dV on the key side.
constexpr int MBQ = 64;               // rows per CTA (4 warps x 16)
constexpr int MBK = 64;               // rows per staged block

// x = hi + lo with hi = x rounded to tf32 (round half away on the magnitude: the integer form
// of cvt.rna.tf32.f32 for finite x, which ptxas expands with an Inf/NaN guard) and lo = x − hi
// exactly; the MMA truncates lo to tf32, an error <= 2^-11·|lo| <= 2^-22·|x|.
__device__ __forceinline__ void tf32_split(float x, uint32_t &hi, uint32_t &lo) {
  const uint32_t h = (__float_as_uint(x) + 0x1000u) & 0xFFFFE000u;
  hi = h;
  lo = __float_as_uint(x - __uint_as_float(h));
}
__device__ __forceinline__ void mma_tf32(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
// rows [r0, r0 + MBK) of X (head slice, times sc) -> hi / lo tiles [MBK][DH + 4]; every
// thread issues all of its float4 loads before the first split (latency overlapped)
template <int DH>
__device__ __forceinline__ void stage_split(const float *__restrict__ X, int D, int hc, int r0, int r1,
                                            float sc, float *xh, float *xl) {
  constexpr int SR = DH + 4, C4 = DH / 4, PER = MBK * C4 / 128;
  float4 v[PER];
#pragma unroll
  for (int u = 0; u < PER; ++u) {
    const int e = threadIdx.x + 128 * u, rr = e / C4, c4 = (e % C4) * 4;
    v[u] = r0 + rr < r1 ? __ldg(reinterpret_cast<const float4 *>(X + long(r0 + rr) * D + hc + c4))
                        : make_float4(0.f, 0.f, 0.f, 0.f);
  }
#pragma unroll
  for (int u = 0; u < PER; ++u) {
    const int e = threadIdx.x + 128 * u, rr = e / C4, c4 = (e % C4) * 4;
    const float x[4] = {v[u].x * sc, v[u].y * sc, v[u].z * sc, v[u].w * sc};
    uint32_t hi[4], lo[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) tf32_split(x[k], hi[k], lo[k]);
    *reinterpret_cast<uint4 *>(xh + rr * SR + c4) = make_uint4(hi[0], hi[1], hi[2], hi[3]);
    *reinterpret_cast<uint4 *>(xl + rr * SR + c4) = make_uint4(lo[0], lo[1], lo[2], lo[3]);
  }
}
// A fragment (16 rows x 8 columns at column c0) of rows ra / rb of X (head slice, times sc)
__device__ __forceinline__ void frag_a(const float *__restrict__ X, int D, int hc, long ra, long rb, int N,
                                       int c0, int t, float sc, uint32_t (&h)[4], uint32_t (&l)[4]) {
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const long r = (q & 1) ? rb : ra;
    const int c = c0 + t + (q >> 1) * 4;
    const float x = r < N ? __ldg(X + r * D + hc + c) * sc : 0.f;
    tf32_split(x, h[q], l[q]);
  }
}
constexpr float LOG2E_F = 1.4426950408889634f;
__device__ __forceinline__ float ex2a(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
constexpr int MNG = 4;                // 8-row groups processed together (independent MMA chains)

// S (or dP) of MNG consecutive 8-column groups starting at block row nt0, A fragments a*[KS],
// B rows from the staged hi / lo tile: per ks the MNG groups' MMAs interleave (independent
// accumulators) so the tensor pipe is not serialised on one accumulator.
template <int KS, int SR>
__device__ __forceinline__ void prod_groups(float (&c)[MNG][4], const uint32_t (&ah)[KS][4], const uint32_t (&al)[KS][4],
                                            const float *bh, const float *bl, int nt0, int g, int t) {
#pragma unroll
  for (int q = 0; q < MNG; ++q) c[q][0] = c[q][1] = c[q][2] = c[q][3] = 0.f;
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
#pragma unroll
    for (int q = 0; q < MNG; ++q) {
      const int o = (nt0 + 8 * q + g) * SR + ks * 8 + t;
      mma_tf32(c[q], ah[ks], __float_as_uint(bh[o]), __float_as_uint(bh[o + 4]));
    }
#pragma unroll
    for (int q = 0; q < MNG; ++q) {
      const int o = (nt0 + 8 * q + g) * SR + ks * 8 + t;
      mma_tf32(c[q], ah[ks], __float_as_uint(bl[o]), __float_as_uint(bl[o + 4]));
    }
#pragma unroll
    for (int q = 0; q < MNG; ++q) {
      const int o = (nt0 + 8 * q + g) * SR + ks * 8 + t;
      mma_tf32(c[q], al[ks], __float_as_uint(bh[o]), __float_as_uint(bh[o + 4]));
    }
  }
}
// C fragment (rows g / g+8, columns 2t / 2t+1 of an 8-wide group) -> A fragment with k = t as
// column 2t and k = t + 4 as column 2t + 1, split hi / lo
__device__ __forceinline__ void c_to_a(const float (&c)[4], uint32_t (&h)[4], uint32_t (&l)[4]) {
  tf32_split(c[0], h[0], l[0]);
  tf32_split(c[2], h[1], l[1]);
  tf32_split(c[1], h[2], l[2]);
  tf32_split(c[3], h[3], l[3]);
}
// acc[n] += A (16 x 8, from c_to_a) x B (8 staged rows nt+2t / nt+2t+1 read as k, columns n·8 + g)
template <int NO, int SR>
__device__ __forceinline__ void prod_rows(float (&acc)[NO][4], const uint32_t (&h)[4], const uint32_t (&l)[4],
                                          const float *bh, const float *bl, int nt, int g, int t) {
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const int o0 = (nt + 2 * t) * SR + n * 8 + g, o1 = o0 + SR;
    mma_tf32(acc[n], h, __float_as_uint(bh[o0]), __float_as_uint(bh[o1]));
  }
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const int o0 = (nt + 2 * t) * SR + n * 8 + g, o1 = o0 + SR;
    mma_tf32(acc[n], h, __float_as_uint(bl[o0]), __float_as_uint(bl[o1]));
  }
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const int o0 = (nt + 2 * t) * SR + n * 8 + g, o1 = o0 + SR;
    mma_tf32(acc[n], l, __float_as_uint(bh[o0]), __float_as_uint(bh[o1]));
  }
}

__device__ __forceinline__ void quad_merge2(float &m, float &l, int &ref) {
#pragma unroll
  for (int o = 1; o <= 2; o <<= 1) {
    const float m2 = __shfl_xor_sync(0xffffffffu, m, o);
    const float l2 = __shfl_xor_sync(0xffffffffu, l, o);
    const int r2 = __shfl_xor_sync(0xffffffffu, ref, o);
    const float mm = fmaxf(m, m2);
    if (mm == -INFINITY) continue;
    const float nl = (m == -INFINITY ? 0.f : l * ex2a(m - mm)) + (m2 == -INFINITY ? 0.f : l2 * ex2a(m2 - mm));
    const int nr = (m == mm && m2 == mm) ? min(ref, r2) : (m2 == mm ? r2 : ref);
    m = mm;
    l = nl;
    ref = nr;
  }
}

template <int DH>
__global__ void __launch_bounds__(128) attn_bwd_q_mma_kernel(const AttnBwdArgs a) {
  constexpr int KS = DH / 8, NO = DH / 8, SR = DH + 4;
  extern __shared__ float smq[];
  float *Kh = smq, *Kl = Kh + MBK * SR, *Vh = Kl + MBK * SR, *Vl = Vh + MBK * SR;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int h = blockIdx.y, hc = h * DH, D = a.D;
  const long q0 = long(blockIdx.x) * MBQ;
  const long qlast = min(q0 + MBQ, long(a.N)) - 1;
  const int ub = __ldg(a.node_off + __ldg(a.node_graph + q0));
  const int ue = __ldg(a.node_off + __ldg(a.node_graph + qlast) + 1);
  const long ra = q0 + warp * 16 + g, rb = ra + 8;
  int kla = 0, kha = 0, klb = 0, khb = 0;
  if (ra < a.N) { const int b = __ldg(a.node_graph + ra); kla = __ldg(a.node_off + b); kha = __ldg(a.node_off + b + 1); }
  if (rb < a.N) { const int b = __ldg(a.node_graph + rb); klb = __ldg(a.node_off + b); khb = __ldg(a.node_off + b + 1); }
  // Q carries log2(e)/√d_h: scores come out in log2 units for ex2
  uint32_t qh[KS][4], ql[KS][4], oh[KS][4], ol[KS][4];
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
    frag_a(a.Q, D, hc, ra, rb, a.N, ks * 8, t, a.scale * LOG2E_F, qh[ks], ql[ks]);
    frag_a(a.dO, D, hc, ra, rb, a.N, ks * 8, t, 1.f, oh[ks], ol[ks]);
  }
  auto inrow = [&](int e, int j) { return (e < 2) ? (j >= kla && j < kha) : (j >= klb && j < khb); };
  // pass 1: row maximum (first arg max) and normaliser over the own graph's keys (log2 units)
  float ma = -INFINITY, mb = -INFINITY, la = 0.f, lb = 0.f;
  int refa = kla, refb = klb;
  for (int t0 = ub; t0 < ue; t0 += MBK) {
    __syncthreads();
    stage_split<DH>(a.K, D, hc, t0, ue, 1.f, Kh, Kl);
    __syncthreads();
    for (int nt0 = 0; nt0 < MBK && t0 + nt0 < ue; nt0 += 8 * MNG) {
      float s[MNG][4];
      prod_groups<KS, SR>(s, qh, ql, Kh, Kl, nt0, g, t);
#pragma unroll
      for (int q = 0; q < MNG; ++q)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int j = t0 + nt0 + 8 * q + 2 * t + (e & 1);
          float &m = (e < 2) ? ma : mb;
          float &l = (e < 2) ? la : lb;
          int &ref = (e < 2) ? refa : refb;
          if (inrow(e, j)) {
            if (s[q][e] > m) {
              l = (m == -INFINITY ? 0.f : l * ex2a(m - s[q][e])) + 1.f;
              m = s[q][e];
              ref = j;
            } else {
              l += ex2a(s[q][e] - m);
            }
          }
        }
    }
  }
  quad_merge2(ma, la, refa);
  quad_merge2(mb, lb, refb);
  const float ila = la > 0.f ? 1.f / la : 0.f, ilb = lb > 0.f ? 1.f / lb : 0.f;
  float dpra = 0.f, dprb = 0.f;                        // dP_ir against the dominant key
  if (ra < a.N)
    for (int c = 0; c < DH; ++c) dpra = fmaf(__ldg(a.dO + ra * D + hc + c), __ldg(a.V + long(refa) * D + hc + c), dpra);
  if (rb < a.N)
    for (int c = 0; c < DH; ++c) dprb = fmaf(__ldg(a.dO + rb * D + hc + c), __ldg(a.V + long(refb) * D + hc + c), dprb);
  // pass 2: D'_i = Σ_j P_ij (dP_ij − dP_ir) (float64); pass 3: dQ_i = Σ_j dS_ij K_j
  double Da = 0.0, Db = 0.0;
  float Dpa = 0.f, Dpb = 0.f;
  float dq[NO][4];
#pragma unroll
  for (int n = 0; n < NO; ++n) dq[n][0] = dq[n][1] = dq[n][2] = dq[n][3] = 0.f;
  for (int pass = 2; pass <= 3; ++pass) {
    for (int t0 = ub; t0 < ue; t0 += MBK) {
      __syncthreads();
      stage_split<DH>(a.K, D, hc, t0, ue, 1.f, Kh, Kl);
      stage_split<DH>(a.V, D, hc, t0, ue, 1.f, Vh, Vl);
      __syncthreads();
      for (int nt0 = 0; nt0 < MBK && t0 + nt0 < ue; nt0 += 8 * MNG) {
        float s[MNG][4], dp[MNG][4];
        prod_groups<KS, SR>(s, qh, ql, Kh, Kl, nt0, g, t);
        prod_groups<KS, SR>(dp, oh, ol, Vh, Vl, nt0, g, t);
#pragma unroll
        for (int q = 0; q < MNG; ++q) {
          float ds[4];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const int j = t0 + nt0 + 8 * q + 2 * t + (e & 1);
            const float p = inrow(e, j) ? ex2a(s[q][e] - (e < 2 ? ma : mb)) * (e < 2 ? ila : ilb) : 0.f;
            const float dd = dp[q][e] - (e < 2 ? dpra : dprb);
            if (pass == 2) {
              if (e < 2) Da = fma(double(p), double(dd), Da);
              else Db = fma(double(p), double(dd), Db);
            }
            ds[e] = p * (dd - (e < 2 ? Dpa : Dpb));
          }
          if (pass == 3) {
            uint32_t dh_[4], dl_[4];
            c_to_a(ds, dh_, dl_);
            prod_rows<NO, SR>(dq, dh_, dl_, Kh, Kl, nt0 + 8 * q, g, t);
          }
        }
      }
    }
    if (pass == 2) {
#pragma unroll
      for (int o = 1; o <= 2; o <<= 1) {
        Da += __shfl_xor_sync(0xffffffffu, Da, o);
        Db += __shfl_xor_sync(0xffffffffu, Db, o);
      }
      Dpa = float(Da);
      Dpb = float(Db);
    }
  }
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const int c = hc + n * 8 + 2 * t;
    if (ra < a.N) *reinterpret_cast<float2 *>(a.dQ + ra * D + c) = make_float2(dq[n][0] * a.scale, dq[n][1] * a.scale);
    if (rb < a.N) *reinterpret_cast<float2 *>(a.dQ + rb * D + c) = make_float2(dq[n][2] * a.scale, dq[n][3] * a.scale);
  }
  if (t == 0) {               // stats in log2 units (m), as the key-side kernel reads them
    if (ra < a.N) *reinterpret_cast<float4 *>(a.stats + (ra * a.heads + h) * 4) = make_float4(ma, la, Dpa, dpra);
    if (rb < a.N) *reinterpret_cast<float4 *>(a.stats + (rb * a.heads + h) * 4) = make_float4(mb, lb, Dpb, dprb);
  }
}

template <int DH>
__global__ void __launch_bounds__(128) attn_bwd_kv_mma_kernel(const AttnBwdArgs a) {
  constexpr int KS = DH / 8, NO = DH / 8, SR = DH + 4;
  extern __shared__ float smk[];
  float *Qh = smk, *Ql = Qh + MBK * SR, *Oh = Ql + MBK * SR, *Ol = Oh + MBK * SR;
  float4 *ss = reinterpret_cast<float4 *>(Ol + MBK * SR);     // [MBK] m (log2), l, D', dP_ir
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int h = blockIdx.y, hc = h * DH, D = a.D;
  const long j0 = long(blockIdx.x) * MBQ;
  const long jlast = min(j0 + MBQ, long(a.N)) - 1;
  const int ub = __ldg(a.node_off + __ldg(a.node_graph + j0));
  const int ue = __ldg(a.node_off + __ldg(a.node_graph + jlast) + 1);
  const long ja = j0 + warp * 16 + g, jb = ja + 8;
  int qla = 0, qha = 0, qlb = 0, qhb = 0;
  if (ja < a.N) { const int b = __ldg(a.node_graph + ja); qla = __ldg(a.node_off + b); qha = __ldg(a.node_off + b + 1); }
  if (jb < a.N) { const int b = __ldg(a.node_graph + jb); qlb = __ldg(a.node_off + b); qhb = __ldg(a.node_off + b + 1); }
  uint32_t kh[KS][4], kl[KS][4], vh[KS][4], vl[KS][4];
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
    frag_a(a.K, D, hc, ja, jb, a.N, ks * 8, t, 1.f, kh[ks], kl[ks]);
    frag_a(a.V, D, hc, ja, jb, a.N, ks * 8, t, 1.f, vh[ks], vl[ks]);
  }
  float dk[NO][4], dv[NO][4];
#pragma unroll
  for (int n = 0; n < NO; ++n) dk[n][0] = dk[n][1] = dk[n][2] = dk[n][3] = dv[n][0] = dv[n][1] = dv[n][2] = dv[n][3] = 0.f;
  for (int t0 = ub; t0 < ue; t0 += MBK) {
    __syncthreads();
    stage_split<DH>(a.Q, D, hc, t0, ue, a.scale * LOG2E_F, Qh, Ql);     // scores in log2 units
    stage_split<DH>(a.dO, D, hc, t0, ue, 1.f, Oh, Ol);
    for (int e = threadIdx.x; e < MBK; e += 128)
      ss[e] = t0 + e < ue ? *reinterpret_cast<const float4 *>(a.stats + (long(t0 + e) * a.heads + h) * 4)
                          : make_float4(0.f, 1.f, 0.f, 0.f);
    __syncthreads();
    for (int nt0 = 0; nt0 < MBK && t0 + nt0 < ue; nt0 += 8 * MNG) {
      // Sᵀ, dPᵀ of the query groups: c0 (ja, query 2t), c1 (ja, 2t+1), c2 (jb, 2t), c3 (jb, 2t+1)
      float s[MNG][4], dp[MNG][4];
      prod_groups<KS, SR>(s, kh, kl, Qh, Ql, nt0, g, t);
      prod_groups<KS, SR>(dp, vh, vl, Oh, Ol, nt0, g, t);
#pragma unroll
      for (int q = 0; q < MNG; ++q) {
        float p[4], ds[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int qi = nt0 + 8 * q + 2 * t + (e & 1), i = t0 + qi;
          const bool in = (e < 2) ? (i >= qla && i < qha) : (i >= qlb && i < qhb);
          const float4 st = ss[qi];
          p[e] = in ? ex2a(s[q][e] - st.x) / st.y : 0.f;
          ds[e] = p[e] * ((dp[q][e] - st.w) - st.z);
        }
        uint32_t ph[4], pl[4], dh_[4], dl_[4];
        c_to_a(p, ph, pl);
        c_to_a(ds, dh_, dl_);
        prod_rows<NO, SR>(dv, ph, pl, Oh, Ol, nt0 + 8 * q, g, t);
        prod_rows<NO, SR>(dk, dh_, dl_, Qh, Ql, nt0 + 8 * q, g, t);
      }
    }
  }
  // Qh carried log2(e)/√d_h; dK = Σ dS Q/√d_h
  const float kfix = 1.f / LOG2E_F;
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const int c = hc + n * 8 + 2 * t;
    if (ja < a.N) {
      *reinterpret_cast<float2 *>(a.dK + ja * D + c) = make_float2(dk[n][0] * kfix, dk[n][1] * kfix);
      *reinterpret_cast<float2 *>(a.dV + ja * D + c) = make_float2(dv[n][0], dv[n][1]);
    }
    if (jb < a.N) {
      *reinterpret_cast<float2 *>(a.dK + jb * D + c) = make_float2(dk[n][2] * kfix, dk[n][3] * kfix);
      *reinterpret_cast<float2 *>(a.dV + jb * D + c) = make_float2(dv[n][2], dv[n][3]);
    }
  }
}
}  // namespace

// ---- launchers ---------------------------------------------------------------------------
// bias-style gradient: out[c] = Σ_r X[r][c] (fixed order)
static int colsum(occu_ctx *ctx, const float *X, long R, float *out, cudaStream_t st) {
  const int D = ctx->cfg.d;
  const int nb = grid_rows(R, ST / 32 * 8, 4 * ctx->num_sms);
  if (ctx->ws.dpart.ensure(size_t(nb) * 2 * D * 8) != cudaSuccess) return -int(cudaErrorMemoryAllocation);
  double *part = reinterpret_cast<double *>(ctx->ws.dpart.ptr);
  OCCU_PROF_BEGIN(ctx, "stack_colsum", st);
  if (D == 64) colsum_kernel<64><<<nb, ST, 0, st>>>(X, R, part);
  else colsum_kernel<128><<<nb, ST, 0, st>>>(X, R, part);
  col_reduce_kernel<<<(D + 127) / 128, 128, 0, st>>>(part, nb, D, D, out, nullptr);
  OCCU_PROF_END(ctx);
  SK_CHECK();
  return 2;
}

int launch_colsum_rows(occu_ctx *ctx, const float *X, long R, float *out, cudaStream_t st) {
  return colsum(ctx, X, R, out, st);
}

static int ln_bwd(occu_ctx *ctx, const float *x, const float *gam, const float *dy, const float *add,
                  float *dx, long R, float *gg, float *gb, cudaStream_t st);
int launch_ln_param_grads(occu_ctx *ctx, const float *x, const float *gam, const float *dy, long R,
                          float *dx_scratch, float *gg, float *gb, cudaStream_t st) {
  return ln_bwd(ctx, x, gam, dy, nullptr, dx_scratch, R, gg, gb, st);
}

// dx = add + LNᵀ(dy) for x = LN input; dγ, dβ into gg, gb.
static int ln_bwd(occu_ctx *ctx, const float *x, const float *gam, const float *dy, const float *add,
                  float *dx, long R, float *gg, float *gb, cudaStream_t st) {
  const int D = ctx->cfg.d;
  const int nb = grid_rows(R, ST / 32 * 8, 4 * ctx->num_sms);
  if (ctx->ws.dpart.ensure(size_t(nb) * 2 * D * 8) != cudaSuccess) return -int(cudaErrorMemoryAllocation);
  double *part = reinterpret_cast<double *>(ctx->ws.dpart.ptr);
  OCCU_PROF_BEGIN(ctx, "stack_ln_bwd", st);
  if (D == 64) ln_bwd_kernel<64><<<nb, ST, 0, st>>>(x, gam, dy, add, dx, R, part);
  else ln_bwd_kernel<128><<<nb, ST, 0, st>>>(x, gam, dy, add, dx, R, part);
  col_reduce_kernel<<<(D + 127) / 128, 128, 0, st>>>(part, nb, D, 2 * D, gg, gb);
  OCCU_PROF_END(ctx);
  SK_CHECK();
  return 2;
}

int launch_mask_dA(const occu_ctx *ctx, const DevCsr &csr, const float *dh, const float *h, float *dA,
                   cudaStream_t st) {
  const occu_config &c = ctx->cfg;
  const long n4 = long(csr.N) * c.d / 4;
  OCCU_PROF_BEGIN(ctx, "stack_mask_dA", st);
  mask_dA_kernel<<<grid_rows(n4, 256, 16 * ctx->num_sms), 256, 0, st>>>(
      dh, h, csr.in_ptr, csr.N, c.d, c.aggr == OCCU_AGGR_MEAN, c.slope, dA);
  OCCU_PROF_END(ctx);
  SK_CHECK();
  return 1;
}

int launch_graphormer_layer_bwd(occu_ctx *ctx, const DevCsr &csr, int j, const float *h_in,
                                const GphSave &sv, const float *dout, float *dh_in, float *scratch,
                                cudaStream_t st) {
  const occu_config &cf = ctx->cfg;
  const GphOff &G = ctx->layout.G[j];
  const float *P = ctx->params.as<float>();
  float *Gr = ctx->grads.as<float>();
  const int D = cf.d, N = csr.N, ts = gph_tslot(cf, j);
  if (N <= 0) return 0;
  const size_t ND = size_t(N) * D;
  float *s1 = scratch, *s2 = scratch + ND, *s3 = scratch + 2 * ND, *s4 = scratch + 3 * ND,
        *s5 = scratch + 4 * ND;
  float *stats = scratch + 5 * ND;                        // [N][heads][4]
  int n = 0, r;
#define SKR(call)                  \
  do {                             \
    if ((r = (call)) < 0) return r; \
    n += r;                        \
  } while (0)
  // FFN: dT = (dout W2) ⊙ [T > 0]; dW2 = doutᵀ T; db2; dX2 = dT W1; dW1 = dTᵀ X2; db1
  SKR(launch_plain_masked_tc(ctx, dout, D, N, 5, ts, nullptr, s1, "stack_gemm_tc", st, sv.T, 0.f));
  SKR(launch_wgrad(ctx, dout, D, sv.T, D, N, Gr + G.F.W2, st, false));
  SKR(colsum(ctx, dout, N, Gr + G.F.b2, st));
  SKR(launch_plain_tc(ctx, s1, D, N, 4, ts, nullptr, s2, "stack_gemm_tc", st));
  SKR(launch_wgrad(ctx, s1, D, sv.X2, D, N, Gr + G.F.W1, st, false));
  SKR(colsum(ctx, s1, N, Gr + G.F.b1, st));
  // dh̄ = dout + LN2ᵀ(dX2)
  SKR(ln_bwd(ctx, sv.Hb, P + G.ln2_g, s2, dout, s3, N, Gr + G.ln2_g, Gr + G.ln2_b, st));
  // dO = dh̄ W_o; dW_o = dh̄ᵀ O; db_o
  SKR(launch_plain_tc(ctx, s3, D, N, 3, ts, nullptr, s2, "stack_gemm_tc", st));
  SKR(launch_wgrad(ctx, s3, D, sv.O, D, N, Gr + G.Wo, st, false));
  SKR(colsum(ctx, s3, N, Gr + G.bo, st));
  // attention backward: dQ -> s1, dK -> s4, dV -> s5
  AttnBwdArgs a;
  a.Q = sv.Q; a.K = sv.K; a.V = sv.V; a.O = sv.O; a.dO = s2;
  a.node_off = csr.node_off; a.node_graph = csr.node_graph;
  a.dQ = s1; a.dK = s4; a.dV = s5; a.stats = stats;
  a.N = N; a.D = D; a.heads = cf.heads;
  const int dh = D / cf.heads;
  a.scale = 1.f / sqrtf(float(dh));
  const dim3 grid((N + ABT - 1) / ABT, cf.heads);
  static const bool simt_attn = getenv("OCCU_ATTN_BWD_SIMT") != nullptr;   // A/B: CUDA-core kernels
  OCCU_PROF_BEGIN(ctx, "stack_attn_bwd", st);
  if (!simt_attn && (dh == 16 || dh == 32)) {
    const dim3 mg((N + MBQ - 1) / MBQ, cf.heads);
    const size_t smq = size_t(4) * MBK * (dh + 4) * 4, smk = smq + size_t(MBK) * 16;
    if (dh == 16) {
      attn_bwd_q_mma_kernel<16><<<mg, 128, smq, st>>>(a);
      attn_bwd_kv_mma_kernel<16><<<mg, 128, smk, st>>>(a);
    } else {
      attn_bwd_q_mma_kernel<32><<<mg, 128, smq, st>>>(a);
      attn_bwd_kv_mma_kernel<32><<<mg, 128, smk, st>>>(a);
    }
  } else switch (dh) {
    case 16: attn_bwd_q_kernel<16><<<grid, ABT, 0, st>>>(a); attn_bwd_kv_kernel<16><<<grid, ABT, 0, st>>>(a); break;
    case 32: attn_bwd_q_kernel<32><<<grid, ABT, 0, st>>>(a); attn_bwd_kv_kernel<32><<<grid, ABT, 0, st>>>(a); break;
    case 64: attn_bwd_q_kernel<64><<<grid, ABT, 0, st>>>(a); attn_bwd_kv_kernel<64><<<grid, ABT, 0, st>>>(a); break;
    default: return -int(cudaErrorInvalidValue);
  }
  OCCU_PROF_END(ctx);
  SK_CHECK();
  n += 2;
  // projections: dW_{q,k,v} = d{Q,K,V}ᵀ X1, biases; dX1 = dQ W_q + dK W_k + dV W_v -> s2
  SKR(launch_wgrad(ctx, s1, D, sv.X1, D, N, Gr + G.Wq, st, false));
  SKR(colsum(ctx, s1, N, Gr + G.bq, st));
  SKR(launch_wgrad(ctx, s4, D, sv.X1, D, N, Gr + G.Wk, st, false));
  SKR(colsum(ctx, s4, N, Gr + G.bk, st));
  SKR(launch_wgrad(ctx, s5, D, sv.X1, D, N, Gr + G.Wv, st, false));
  SKR(colsum(ctx, s5, N, Gr + G.bv, st));
  SKR(launch_plain_tc(ctx, s1, D, N, 0, ts, nullptr, s2, "stack_gemm_tc", st));
  SKR(launch_plain_tc(ctx, s4, D, N, 1, ts, s2, s2, "stack_gemm_tc", st));
  SKR(launch_plain_tc(ctx, s5, D, N, 2, ts, s2, s2, "stack_gemm_tc", st));
  // dH = dh̄ + LN1ᵀ(dX1)
  SKR(ln_bwd(ctx, h_in, P + G.ln1_g, s2, s3, dh_in, N, Gr + G.ln1_g, Gr + G.ln1_b, st));
#undef SKR
  return n;
}

}  // namespace occu
