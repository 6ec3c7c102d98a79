// FP32 CUDA-core (SIMT) kernels for the ANEE hot path on sm_100a.
//
// Forward, per layer (DESIGN.md §1 rows a2-a6; P141-P151 with readings R1-R9):
//   node_gemm   : h̄ = LReLU(h W_uᵀ), p = h̄·a_s, q = h̄·a_d                    (a2)
//   edge_fwd    : z = W_e e ; e' = σ((p[s]+q[t]) z) ; g = softmax_c(W_m e')   (a3, a4)
//   gather_segsum: h[t] = LReLU(Σ_{k∈seg(t)} g_k ⊙ h̄[s_k])  (warp per node)   (a5, a6)
// then readout_head (a7, a8).  Backward (a9, a10) and Adam (a12) follow the
// hand derivation in SURVEY §8(c) "Step BW"; every reduction has a fixed order
// (no atomics), so results are bitwise reproducible.
//
// Tiling: 64-row tiles, 256 threads as 16 (tx) x 16 (ty); thread owns rows
// ty*4..ty*4+3 and columns {tx*4+j, 64+tx*4+j}.  The whole weight matrix sits
// in shared memory (d <= 128), persistent CTAs loop over tiles.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>

#include "occu_internal.h"

namespace occu {
namespace {

constexpr int BM = 64;
constexpr int NT = 256;

__device__ __forceinline__ float lrelu(float x, float s) { return x > 0.f ? x : s * x; }
__device__ __forceinline__ float lrelu_grad_from_out(float y, float s) { return y > 0.f ? 1.f : s; }
__device__ __forceinline__ float sigmoidf_(float x) { return 1.f / (1.f + expf(-x)); }
__device__ __forceinline__ float ex2f_fast(float x) {     // MUFU.EX2 (~2 ulp); ex2(-inf) = 0
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
// Element i of an FP32 or (BF = true) BF16 stored activation (OCCU_BF16 training, R28).
template <bool BF> __device__ __forceinline__ float ld_act(const void *base, long i) {
  if constexpr (BF)
    return __uint_as_float(uint32_t(__ldg(reinterpret_cast<const unsigned short *>(base) + i)) << 16);
  else
    return __ldg(reinterpret_cast<const float *>(base) + i);
}

__device__ __forceinline__ float hsum16(float v) {   // sum over the 16 lanes sharing ty
  v += __shfl_xor_sync(0xffffffffu, v, 1);
  v += __shfl_xor_sync(0xffffffffu, v, 2);
  v += __shfl_xor_sync(0xffffffffu, v, 4);
  v += __shfl_xor_sync(0xffffffffu, v, 8);
  return v;
}
// Cancellation-prone dot products (softmax backward <g, dg>, dα = <dy, z>) are
// accumulated in float64 (a few hundred DFMA per edge).
__device__ __forceinline__ double hsum16d(double v) {
  v += __shfl_xor_sync(0xffffffffu, v, 1);
  v += __shfl_xor_sync(0xffffffffu, v, 2);
  v += __shfl_xor_sync(0xffffffffu, v, 4);
  v += __shfl_xor_sync(0xffffffffu, v, 8);
  return v;
}
__device__ __forceinline__ float hmax16(float v) {
  v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 1));
  v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 2));
  v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 4));
  v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 8));
  return v;
}

// Column owned by (tx, j): D=128 -> tx*4+j (j<4) and 64+tx*4+(j-4); D=64 -> tx*4+j.
template <int D> __device__ __forceinline__ int colof(int tx, int j) {
  return (j < 4) ? tx * 4 + j : 64 + tx * 4 + (j - 4);
}
template <int D> struct Tn { static constexpr int v = D / 16; };

// Load W into smem as Ws[k][n] (row length D).  TRANS: W is [D][K] and
// Ws[k][n] = W[n][k] (for y = x Wᵀ); otherwise W is [K][D] and Ws = W.
template <int D, bool TRANS>
__device__ void load_weights(float *Ws, const float *__restrict__ W, int K) {
  if (TRANS) {
    for (int idx = threadIdx.x; idx < K * D; idx += NT) {
      const int n = idx / K, k = idx % K;        // coalesced read of W[n][k]
      Ws[k * D + n] = W[idx];
    }
  } else {
    for (int idx = threadIdx.x; idx < K * D; idx += NT) Ws[idx] = W[idx];
  }
}

// Load `rows` x K (row-major, K % 4 == 0) rows starting at row0 into As with
// row stride S = K + 4; rows beyond `nrows` are zero.
__device__ void load_rows(float *As, const float *__restrict__ A, long row0, int nrows, int K) {
  const int S = K + 4, kq = K / 4;
  for (int idx = threadIdx.x; idx < BM * kq; idx += NT) {
    const int r = idx / kq, c = (idx % kq) * 4;
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (r < nrows) v = __ldg(reinterpret_cast<const float4 *>(A + (row0 + r) * K + c));
    *reinterpret_cast<float4 *>(As + r * S + c) = v;
  }
}

// acc[i][j] += Σ_k As[row_i][k] * Ws[k][col_j], rows ty*4+i, K % 4 == 0.
template <int D>
__device__ __forceinline__ void gemm_tile(const float *As, int K, const float *Ws,
                                          float (&acc)[4][Tn<D>::v], int tx, int ty) {
  constexpr int TN = Tn<D>::v;
  const int S = K + 4;
  for (int k = 0; k < K; k += 4) {
    float4 a[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) a[i] = *reinterpret_cast<const float4 *>(As + (ty * 4 + i) * S + k);
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      float b[TN];
      const float *w = Ws + (k + kk) * D;
      const float4 b0 = *reinterpret_cast<const float4 *>(w + tx * 4);
      b[0] = b0.x; b[1] = b0.y; b[2] = b0.z; b[3] = b0.w;
      if (TN == 8) {
        const float4 b1 = *reinterpret_cast<const float4 *>(w + 64 + tx * 4);
        b[4 % TN] = b1.x; b[5 % TN] = b1.y; b[6 % TN] = b1.z; b[7 % TN] = b1.w;
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float av = kk == 0 ? a[i].x : kk == 1 ? a[i].y : kk == 2 ? a[i].z : a[i].w;
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(av, b[j], acc[i][j]);
      }
    }
  }
}

template <int D> __device__ __forceinline__ void zero_acc(float (&acc)[4][Tn<D>::v]) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < Tn<D>::v; ++j) acc[i][j] = 0.f;
}

// Store a row-slice of 4-column groups (float4) for row r of a [*, D] matrix.
template <int D>
__device__ __forceinline__ void store_row(float *dst, const float (&v)[Tn<D>::v], int tx) {
  *reinterpret_cast<float4 *>(dst + tx * 4) = make_float4(v[0], v[1], v[2], v[3]);
  if (Tn<D>::v == 8)
    *reinterpret_cast<float4 *>(dst + 64 + tx * 4) =
        make_float4(v[4 % Tn<D>::v], v[5 % Tn<D>::v], v[6 % Tn<D>::v], v[7 % Tn<D>::v]);
}
template <int D>
__device__ __forceinline__ void load_row(const float *src, float (&v)[Tn<D>::v], int tx) {
  const float4 a = __ldg(reinterpret_cast<const float4 *>(src + tx * 4));
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  if (Tn<D>::v == 8) {
    const float4 b = __ldg(reinterpret_cast<const float4 *>(src + 64 + tx * 4));
    v[4 % Tn<D>::v] = b.x; v[5 % Tn<D>::v] = b.y; v[6 % Tn<D>::v] = b.z; v[7 % Tn<D>::v] = b.w;
  }
}

// ---------------------------------------------------------------------------
// a2: node transform.  MODE 0: h̄ = LReLU(A Wᵀ), p, q (forward).
//                      MODE 1: C = A W (plain GEMM, backward dh_prev = dP W_u).
// ---------------------------------------------------------------------------
template <int D, int MODE>
__global__ void __launch_bounds__(NT) node_gemm_kernel(const float *__restrict__ A, int K,
                                                       const float *__restrict__ W,
                                                       const float *__restrict__ a_s,
                                                       const float *__restrict__ a_d, int N,
                                                       float slope, float *__restrict__ out,
                                                       float *__restrict__ p,
                                                       float *__restrict__ q) {
  extern __shared__ __align__(16) float smem[];
  float *Ws = smem;                 // [K][D]
  float *As = Ws + K * D;           // [BM][K+4]
  constexpr int TN = Tn<D>::v;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  load_weights<D, MODE == 0>(Ws, W, K);
  float as_[TN], ad_[TN];
  if (MODE == 0) {
#pragma unroll
    for (int j = 0; j < TN; ++j) {
      as_[j] = a_s[colof<D>(tx, j)];
      ad_[j] = a_d[colof<D>(tx, j)];
    }
  }
  const int tiles = (N + BM - 1) / BM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long r0 = long(tile) * BM;
    const int nrows = min(BM, int(N - r0));
    __syncthreads();
    load_rows(As, A, r0, nrows, K);
    __syncthreads();
    float acc[4][TN];
    zero_acc<D>(acc);
    gemm_tile<D>(As, K, Ws, acc, tx, ty);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = ty * 4 + i;
      float v[TN];
      float pp = 0.f, qq = 0.f;
#pragma unroll
      for (int j = 0; j < TN; ++j) {
        v[j] = MODE == 0 ? lrelu(acc[i][j], slope) : acc[i][j];
        if (MODE == 0) {
          pp = fmaf(v[j], as_[j], pp);
          qq = fmaf(v[j], ad_[j], qq);
        }
      }
      if (MODE == 0) {
        pp = hsum16(pp);
        qq = hsum16(qq);
      }
      if (r < nrows) {
        store_row<D>(out + (r0 + r) * D, v, tx);
        if (MODE == 0 && tx == 0) {
          p[r0 + r] = pp;
          q[r0 + r] = qq;
        }
      }
    }
  }
}

// ---------------------------------------------------------------------------
// a3 + a4: edge transform and channel softmax gate, edges in in-CSR order.
// ---------------------------------------------------------------------------
template <int D>
__global__ void __launch_bounds__(NT) edge_fwd_kernel(
    const float *__restrict__ e_in, int Ke, const float *__restrict__ W_e,
    const float *__restrict__ W_m, const float *__restrict__ p, const float *__restrict__ q,
    const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst, int E,
    float *__restrict__ e_out, float *__restrict__ g_out) {
  extern __shared__ __align__(16) float smem[];
  float *Wes = smem;                // [Ke][D]  (W_eᵀ)
  float *Wms = Wes + Ke * D;        // [D][D]   (W_mᵀ)
  float *As = Wms + D * D;          // [BM][Ke+4]
  float *Es = As + BM * (Ke + 4);   // [BM][D+4]
  float *alpha = Es + BM * (D + 4); // [BM]
  constexpr int TN = Tn<D>::v;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  load_weights<D, true>(Wes, W_e, Ke);
  load_weights<D, true>(Wms, W_m, D);
  const int tiles = (E + BM - 1) / BM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long k0 = long(tile) * BM;
    const int nrows = min(BM, int(E - k0));
    __syncthreads();
    load_rows(As, e_in, k0, nrows, Ke);
    if (threadIdx.x < BM) {
      const int r = threadIdx.x;
      alpha[r] = r < nrows ? p[in_src[k0 + r]] + q[in_dst[k0 + r]] : 0.f;   // R1
    }
    __syncthreads();
    float acc[4][TN];
    zero_acc<D>(acc);
    gemm_tile<D>(As, Ke, Wes, acc, tx, ty);                                  // z = W_e e
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = ty * 4 + i;
      const float al = alpha[r];
      float v[TN];
#pragma unroll
      for (int j = 0; j < TN; ++j) v[j] = sigmoidf_(al * acc[i][j]);          // e' (R2, R3)
      store_row<D>(Es + r * (D + 4), v, tx);
      if (e_out && r < nrows) store_row<D>(e_out + (k0 + r) * D, v, tx);
    }
    __syncthreads();
    zero_acc<D>(acc);
    gemm_tile<D>(Es, D, Wms, acc, tx, ty);                                   // v = W_m e'
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = ty * 4 + i;
      float mx = -INFINITY;
#pragma unroll
      for (int j = 0; j < TN; ++j) mx = fmaxf(mx, acc[i][j]);
      mx = hmax16(mx);
      float v[TN], s = 0.f;
#pragma unroll
      for (int j = 0; j < TN; ++j) {
        v[j] = expf(acc[i][j] - mx);
        s += v[j];
      }
      s = hsum16(s);
#pragma unroll
      for (int j = 0; j < TN; ++j) v[j] = v[j] / s;                           // g (R4 reading A)
      if (r < nrows) store_row<D>(g_out + (k0 + r) * D, v, tx);
    }
  }
}

template <int V>
__device__ __forceinline__ void store_row(float *dst, const float (&v)[V]) {
  if constexpr (V == 4) {
    *reinterpret_cast<float4 *>(dst) = make_float4(v[0], v[1], v[2], v[3]);
  } else if constexpr (V == 8) {
    *reinterpret_cast<float4 *>(dst) = make_float4(v[0], v[1], v[2], v[3]);
    *reinterpret_cast<float4 *>(dst + 4) = make_float4(v[4 % V], v[5 % V], v[6 % V], v[7 % V]);
  } else {
#pragma unroll
    for (int c = 0; c < V; ++c) dst[c] = v[c];
  }
}

// ---------------------------------------------------------------------------
// a5 + a6: gather + deterministic segmented sum, warp per destination node.
// Lane l owns channels [l*V, l*V+V), V = D/32; edges summed in ascending k.
// ---------------------------------------------------------------------------
template <int D, bool RP>
__global__ void __launch_bounds__(NT) gather_segsum_kernel(
    const float *__restrict__ g, const float *__restrict__ hbar,
    const int32_t *__restrict__ in_ptr, const int32_t *__restrict__ in_src, int N, int mean,
    float slope, float *__restrict__ h_out, const int32_t *__restrict__ node_graph,
    float *__restrict__ rpart) {
  // A warp owns NPW consecutive destination nodes (a "chunk"), i.e. the contiguous
  // in-CSR edge range [in_ptr[t0], in_ptr[t0+NPW]); edges are consumed in ascending
  // order, four gathered rows in flight at a time, and each node's sum is flushed when
  // the edge index crosses its segment end (fixed order: identical to a per-node loop).
  // Last layer (rpart != null): the flushed rows h_u are also summed per graph inside
  // the chunk, in ascending u, and graph b's chunk partial is stored at row
  // min(u1 - 1, t0 + NPW - 1) of rpart (its last node in the chunk) for
  // readout_head_kernel (a7); h_out may then be null (inference never re-reads h_L).
  constexpr int V = D / 32;
  constexpr int NPW = 8;
  const int lane = threadIdx.x & 31;
  const long warps = (long(gridDim.x) * NT) / 32;
  for (long t0 = (blockIdx.x * long(NT) + threadIdx.x) / 32 * NPW; t0 < N; t0 += warps * NPW) {
    const int nn = int(min(long(NPW), N - t0));
    const int ptr_l = lane <= nn ? in_ptr[t0 + lane] : 0;      // in_ptr[t0 .. t0+nn]
    const int gr_l = (RP && lane < nn) ? node_graph[t0 + lane] : -1;
    const int e_beg = __shfl_sync(0xffffffffu, ptr_l, 0);
    const int e_end = __shfl_sync(0xffffffffu, ptr_l, nn);
    int node = 0;                                               // local node index
    int seg_end = __shfl_sync(0xffffffffu, ptr_l, 1);
    float acc[V], racc[V];
#pragma unroll
    for (int c = 0; c < V; ++c) acc[c] = racc[c] = 0.f;
#define OCCU_FLUSH_NODE(nd)                                                                  \
  do {                                                                                       \
    const int deg_ = __shfl_sync(0xffffffffu, ptr_l, (nd) + 1) - __shfl_sync(0xffffffffu, ptr_l, (nd)); \
    if constexpr (!RP) {                                                                     \
      float *o_ = h_out + (t0 + (nd)) * D + lane * V;                                        \
      _Pragma("unroll") for (int c = 0; c < V; ++c) {                                        \
        float a_ = acc[c];                                                                   \
        if (mean) a_ = a_ / float(deg_ > 0 ? deg_ : 1);                                      \
        o_[c] = lrelu(a_, slope);                                                            \
        acc[c] = 0.f;                                                                        \
      }                                                                                      \
    } else {                                                                                 \
      float o_[V];                                                                           \
      _Pragma("unroll") for (int c = 0; c < V; ++c) {                                        \
        float a_ = acc[c];                                                                   \
        if (mean) a_ = a_ / float(deg_ > 0 ? deg_ : 1);                                      \
        o_[c] = lrelu(a_, slope);                                                            \
        acc[c] = 0.f;                                                                        \
      }                                                                                      \
      if (h_out) store_row<V>(h_out + (t0 + (nd)) * D + lane * V, o_);                       \
      const int gcur_ = __shfl_sync(0xffffffffu, gr_l, (nd));                                \
      const int gnxt_ = __shfl_sync(0xffffffffu, gr_l, ((nd) + 1) & 31);                     \
      _Pragma("unroll") for (int c = 0; c < V; ++c) racc[c] += o_[c];                        \
      if ((nd) + 1 >= nn || gnxt_ != gcur_) {                                                \
        store_row<V>(rpart + (t0 + (nd)) * D + lane * V, racc);                              \
        _Pragma("unroll") for (int c = 0; c < V; ++c) racc[c] = 0.f;                         \
      }                                                                                      \
    }                                                                                        \
  } while (0)
    for (int base = e_beg; base < e_end; base += 32) {
      const int cnt = min(32, e_end - base);
      const int s_l = lane < cnt ? in_src[base + lane] : 0;
      for (int j = 0; j < cnt; j += 4) {
        float gv[4][V], hv[4][V];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int s = __shfl_sync(0xffffffffu, s_l, (j + u) & 31);
          if (j + u < cnt) {
            const float *gr = g + long(base + j + u) * D + lane * V;
            const float *hr = hbar + long(s) * D + lane * V;
            if (V == 4) {
              const float4 a = __ldg(reinterpret_cast<const float4 *>(gr));
              const float4 b2 = __ldg(reinterpret_cast<const float4 *>(hr));
              gv[u][0] = a.x; gv[u][1 % V] = a.y; gv[u][2 % V] = a.z; gv[u][3 % V] = a.w;
              hv[u][0] = b2.x; hv[u][1 % V] = b2.y; hv[u][2 % V] = b2.z; hv[u][3 % V] = b2.w;
            } else {
#pragma unroll
              for (int c = 0; c < V; ++c) {
                gv[u][c] = __ldg(gr + c);
                hv[u][c] = __ldg(hr + c);
              }
            }
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          if (j + u < cnt) {
            const int k = base + j + u;
            while (k >= seg_end) {                  // warp-uniform
              OCCU_FLUSH_NODE(node);
              ++node;
              seg_end = __shfl_sync(0xffffffffu, ptr_l, node + 1);
            }
#pragma unroll
            for (int c = 0; c < V; ++c) acc[c] = fmaf(gv[u][c], hv[u][c], acc[c]);
          }
        }
      }
    }
    for (; node < nn; ++node) OCCU_FLUSH_NODE(node);   // remaining (and in-degree-0) nodes
#undef OCCU_FLUSH_NODE
  }
}

// Variant with deeper memory-level parallelism (same arithmetic and summation order
// as gather_segsum_kernel): persistent warps walk chunks of NPW destinations; each
// group issues G gathered (g, h̄[s]) row pairs unconditionally (indices clamped into
// the chunk, surplus rows are never accumulated), and the next chunk's in_ptr /
// in_src words are requested while the current chunk is summed.
template <int V, bool BF>
__device__ __forceinline__ void load_row(const void *base, long row, int D, int lane, float (&v)[V]) {
  if constexpr (BF) {
    const __nv_bfloat16 *p = reinterpret_cast<const __nv_bfloat16 *>(base) + row * D + lane * V;
    if constexpr (V == 4) {
      const uint2 x = __ldg(reinterpret_cast<const uint2 *>(p));
      const float2 a = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162 *>(&x.x));
      const float2 b = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162 *>(&x.y));
      v[0] = a.x; v[1 % V] = a.y; v[2 % V] = b.x; v[3 % V] = b.y;
    } else {
#pragma unroll
      for (int c = 0; c < V; c += 2) {
        const uint32_t x = __ldg(reinterpret_cast<const unsigned int *>(p + c));
        const float2 a = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162 *>(&x));
        v[c] = a.x; v[(c + 1) % V] = a.y;
      }
    }
  } else {
    const float *p = reinterpret_cast<const float *>(base) + row * D + lane * V;
    if constexpr (V == 4) {
      const float4 a = __ldg(reinterpret_cast<const float4 *>(p));
      v[0] = a.x; v[1 % V] = a.y; v[2 % V] = a.z; v[3 % V] = a.w;
    } else if constexpr (V == 8) {
      const float4 a = __ldg(reinterpret_cast<const float4 *>(p));
      const float4 b = __ldg(reinterpret_cast<const float4 *>(p + 4));
      v[0] = a.x; v[1 % V] = a.y; v[2 % V] = a.z; v[3 % V] = a.w;
      v[4 % V] = b.x; v[5 % V] = b.y; v[6 % V] = b.z; v[7 % V] = b.w;
    } else {
#pragma unroll
      for (int c = 0; c < V; ++c) v[c] = __ldg(p + c);
    }
  }
}
// A lane's V-channel slice of a stored row, kept in its storage type until use (BF16
// rows stay packed: half the registers per row in flight).
template <int V, bool BF> struct RawRow;
template <> struct RawRow<4, false> {
  float4 v;
  __device__ __forceinline__ void load(const void *b, long row, int D, int lane) {
    v = __ldg(reinterpret_cast<const float4 *>(reinterpret_cast<const float *>(b) + row * D + lane * 4));
  }
  __device__ __forceinline__ void get(float (&o)[4]) const { o[0] = v.x; o[1] = v.y; o[2] = v.z; o[3] = v.w; }
};
// d = 256: a lane's 8 channels = two float4 (one 1 KB row per warp, fully coalesced)
template <> struct RawRow<8, false> {
  float4 v0, v1;
  __device__ __forceinline__ void load(const void *b, long row, int D, int lane) {
    const float4 *p = reinterpret_cast<const float4 *>(reinterpret_cast<const float *>(b) + row * D + lane * 8);
    v0 = __ldg(p);
    v1 = __ldg(p + 1);
  }
  __device__ __forceinline__ void get(float (&o)[8]) const {
    o[0] = v0.x; o[1] = v0.y; o[2] = v0.z; o[3] = v0.w;
    o[4] = v1.x; o[5] = v1.y; o[6] = v1.z; o[7] = v1.w;
  }
};
template <> struct RawRow<8, true> {
  uint4 v;
  __device__ __forceinline__ void load(const void *b, long row, int D, int lane) {
    v = __ldg(reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(b) + row * D + lane * 8));
  }
  __device__ __forceinline__ void get(float (&o)[8]) const {
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      o[2 * i] = __uint_as_float(w[i] << 16);
      o[2 * i + 1] = __uint_as_float(w[i] & 0xFFFF0000u);
    }
  }
};
template <> struct RawRow<2, false> {
  float2 v;
  __device__ __forceinline__ void load(const void *b, long row, int D, int lane) {
    v = __ldg(reinterpret_cast<const float2 *>(reinterpret_cast<const float *>(b) + row * D + lane * 2));
  }
  __device__ __forceinline__ void get(float (&o)[2]) const { o[0] = v.x; o[1] = v.y; }
};
template <> struct RawRow<4, true> {
  uint2 v;
  __device__ __forceinline__ void load(const void *b, long row, int D, int lane) {
    v = __ldg(reinterpret_cast<const uint2 *>(reinterpret_cast<const __nv_bfloat16 *>(b) + row * D + lane * 4));
  }
  __device__ __forceinline__ void get(float (&o)[4]) const {
    o[0] = __uint_as_float(v.x << 16); o[1] = __uint_as_float(v.x & 0xFFFF0000u);
    o[2] = __uint_as_float(v.y << 16); o[3] = __uint_as_float(v.y & 0xFFFF0000u);
  }
};
template <> struct RawRow<2, true> {
  uint32_t v;
  __device__ __forceinline__ void load(const void *b, long row, int D, int lane) {
    v = __ldg(reinterpret_cast<const unsigned int *>(reinterpret_cast<const __nv_bfloat16 *>(b) + row * D + lane * 2));
  }
  __device__ __forceinline__ void get(float (&o)[2]) const {
    o[0] = __uint_as_float(v << 16); o[1] = __uint_as_float(v & 0xFFFF0000u);
  }
};

template <int V, bool BF>
__device__ __forceinline__ void store_row_t(void *base, long row, int D, int lane, const float (&v)[V]) {
  if constexpr (BF) {
    __nv_bfloat16 *p = reinterpret_cast<__nv_bfloat16 *>(base) + row * D + lane * V;
    uint32_t w[V / 2];
#pragma unroll
    for (int c = 0; c < V; c += 2) {
      const __nv_bfloat162 h = __floats2bfloat162_rn(v[c], v[c + 1]);
      w[c / 2] = *reinterpret_cast<const uint32_t *>(&h);
    }
    if constexpr (V == 8) *reinterpret_cast<uint4 *>(p) = make_uint4(w[0], w[1 % (V / 2)], w[2 % (V / 2)], w[3 % (V / 2)]);
    else if constexpr (V == 4) *reinterpret_cast<uint2 *>(p) = make_uint2(w[0], w[1 % (V / 2)]);
    else *reinterpret_cast<uint32_t *>(p) = w[0];
  } else {
    store_row<V>(reinterpret_cast<float *>(base) + row * D + lane * V, v);
  }
}

// ---------------------------------------------------------------------------
// Hub destinations (in-degree > HUB_DEG, e.g. §8(d)'s skew benchmark): one warp would walk the
// whole segment alone, so it is split into 64-edge units first — hub_partial_kernel sums each
// unit's share of a hub segment (ascending edge order, warp per unit, slot 0 = the unit's
// first destination, slot 1 = its last), hub_merge_kernel adds a hub's unit partials in unit
// order into the slot of its first unit, and gather_segsum_v2 takes that sum for the node
// instead of walking its edges.  Fixed order throughout (deterministic, atomic-free).
constexpr int HUB_DEG = 256, HUB_UB = 64;

template <int D, bool BF>
__global__ void __launch_bounds__(NT) hub_partial_kernel(
    const void *__restrict__ g, const void *__restrict__ hbar, const int32_t *__restrict__ in_ptr,
    const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst, int E,
    float *__restrict__ part) {
  constexpr int V = D / 32, G = 4;
  const int lane = threadIdx.x & 31;
  const long nw = (long(gridDim.x) * NT) / 32;
  const long units = (long(E) + HUB_UB - 1) / HUB_UB;
  for (long u = (blockIdx.x * long(NT) + threadIdx.x) / 32; u < units; u += nw) {
    const int kb = int(u * HUB_UB), ke = int(min(long(E), u * HUB_UB + HUB_UB));
    const int t0 = __ldg(in_dst + kb), t1 = __ldg(in_dst + ke - 1);
    for (int slot = 0; slot < 2; ++slot) {
      const int t = slot ? t1 : t0;
      if (slot && t1 == t0) break;
      const int sb = __ldg(in_ptr + t), se = __ldg(in_ptr + t + 1);
      if (se - sb <= HUB_DEG) continue;
      const int a = max(kb, sb), b = min(ke, se);
      float acc[V];
#pragma unroll
      for (int c = 0; c < V; ++c) acc[c] = 0.f;
      for (int base = a; base < b; base += 32) {
        const int cnt = min(32, b - base);
        const int s_l = lane < cnt ? __ldg(in_src + base + lane) : 0;
        for (int j = 0; j < cnt; j += G) {
          RawRow<V, BF> gr[G], hr[G];
#pragma unroll
          for (int q = 0; q < G; ++q) {
            const int kk = min(j + q, cnt - 1);
            gr[q].load(g, long(base + kk), D, lane);
            hr[q].load(hbar, long(__shfl_sync(0xffffffffu, s_l, kk)), D, lane);
          }
#pragma unroll
          for (int q = 0; q < G; ++q)
            if (j + q < cnt) {
              float gv[V], hv[V];
              gr[q].get(gv);
              hr[q].get(hv);
#pragma unroll
              for (int c = 0; c < V; ++c) acc[c] = fmaf(gv[c], hv[c], acc[c]);
            }
        }
      }
      store_row<V>(part + (u * 2 + slot) * D + lane * V, acc);
    }
  }
}

template <int D>
__global__ void __launch_bounds__(NT) hub_merge_kernel(const int32_t *__restrict__ in_ptr,
                                                       const int32_t *__restrict__ in_dst, int E,
                                                       float *__restrict__ part) {
  constexpr int V = D / 32;
  const int lane = threadIdx.x & 31;
  const long nw = (long(gridDim.x) * NT) / 32;
  const long units = (long(E) + HUB_UB - 1) / HUB_UB;
  for (long u = (blockIdx.x * long(NT) + threadIdx.x) / 32; u < units; u += nw) {
    const int kb = int(u * HUB_UB), ke = int(min(long(E), u * HUB_UB + HUB_UB));
    const int t0 = __ldg(in_dst + kb), t1 = __ldg(in_dst + ke - 1);
    for (int slot = 0; slot < 2; ++slot) {
      const int t = slot ? t1 : t0;
      if (slot && t1 == t0) break;
      const int sb = __ldg(in_ptr + t), se = __ldg(in_ptr + t + 1);
      if (se - sb <= HUB_DEG || sb / HUB_UB != u) continue;   // merged by its first unit only
      float acc[V];
#pragma unroll
      for (int c = 0; c < V; ++c) acc[c] = part[(u * 2 + slot) * D + lane * V + c];
      for (long u2 = u + 1; u2 <= (se - 1) / HUB_UB; ++u2)     // later units: t is their first dst
#pragma unroll
        for (int c = 0; c < V; ++c) acc[c] += part[(u2 * 2) * D + lane * V + c];
      store_row<V>(part + (u * 2 + slot) * D + lane * V, acc);
    }
  }
}

// HB: training forward — also write the sign bits of h (hbits); a separate instantiation so that
// the inference kernels carry none of its registers
template <int D, int G, bool RP, bool BF = false, bool PF = false, bool HB = false>
__global__ void __launch_bounds__(NT, (BF ? G <= 8 : (G == 4 && !RP && !HB)) ? 4 : 3) gather_segsum_v2_kernel(
    const void *__restrict__ g, const void *__restrict__ hbar,
    const int32_t *__restrict__ in_ptr, const int32_t *__restrict__ in_src, int N, int mean,
    float slope, void *__restrict__ h_out, const int32_t *__restrict__ node_graph,
    float *__restrict__ rpart, const float *__restrict__ hubsum = nullptr,
    const int32_t *__restrict__ in_dst = nullptr, uint32_t *__restrict__ hbits = nullptr) {
  constexpr int V = D / 32;
  constexpr int NPW = 8;
  const int lane = threadIdx.x & 31;
  const long nw = (long(gridDim.x) * NT) / 32;
  long t0 = (blockIdx.x * long(NT) + threadIdx.x) / 32 * NPW;
  pdl_trigger();
  pdl_wait();
  if (t0 >= N) return;
  auto load_ptr = [&](long t) {
    const int n = int(min(long(NPW), N - t));
    return lane <= n ? __ldg(in_ptr + t + lane) : 0;
  };
  int ptr_l = load_ptr(t0);
  int s_first = 0;
  {
    const int eb = __shfl_sync(0xffffffffu, ptr_l, 0);
    const int n = int(min(long(NPW), N - t0));
    const int ee = __shfl_sync(0xffffffffu, ptr_l, n);
    s_first = eb + lane < ee ? __ldg(in_src + eb + lane) : 0;
  }
  for (; t0 < N; t0 += nw * NPW) {
    const int nn = int(min(long(NPW), N - t0));
    const long t1 = t0 + nw * NPW;
    const int ptr_n = t1 < N ? load_ptr(t1) : 0;             // next chunk, in flight now
    const int gr_l = (RP && lane < nn) ? __ldg(node_graph + t0 + lane) : -1;
    const int e_beg = __shfl_sync(0xffffffffu, ptr_l, 0);
    const int e_end = __shfl_sync(0xffffffffu, ptr_l, nn);
    int node = 0;
    int seg_end = __shfl_sync(0xffffffffu, ptr_l, 1);
    float acc[V], racc[V];
#pragma unroll
    for (int c = 0; c < V; ++c) acc[c] = racc[c] = 0.f;
    auto flush = [&](int nd) {
      const int deg = __shfl_sync(0xffffffffu, ptr_l, nd + 1) - __shfl_sync(0xffffffffu, ptr_l, nd);
      float o[V];
#pragma unroll
      for (int c = 0; c < V; ++c) {
        float x = acc[c];
        if (mean) x = x / float(deg > 0 ? deg : 1);
        o[c] = lrelu(x, slope);
        acc[c] = 0.f;
      }
      if (!RP || h_out) store_row_t<V, BF>(h_out, t0 + nd, D, lane, o);
      if constexpr (HB) {      // word c, bit l: channel V·l + c is positive (LReLU' = 1)
        uint32_t mine = 0u;
#pragma unroll
        for (int c = 0; c < V; ++c) {
          const uint32_t m = __ballot_sync(0xffffffffu, o[c] > 0.f);
          if (lane == c) mine = m;
        }
        if (lane < V) hbits[(t0 + nd) * V + lane] = mine;
      }
      if (RP) {
        const int gc = __shfl_sync(0xffffffffu, gr_l, nd);
        const int gn = __shfl_sync(0xffffffffu, gr_l, (nd + 1) & 31);
#pragma unroll
        for (int c = 0; c < V; ++c) racc[c] += o[c];
        if (nd + 1 >= nn || gn != gc) {
          store_row<V>(rpart + (t0 + nd) * D + lane * V, racc);
#pragma unroll
          for (int c = 0; c < V; ++c) racc[c] = 0.f;
        }
      }
    };
    int s_l = s_first;
    int s_next = 0;
    bool next_src_issued = false;
    bool slow = false;
    if (hubsum) {     // a hub in this chunk: nodes one by one, hubs from their merged unit sums
      const int deg_l = __shfl_down_sync(0xffffffffu, ptr_l, 1) - ptr_l;
      slow = __ballot_sync(0xffffffffu, lane < nn && deg_l > HUB_DEG) != 0u;
    }
    if (slow) {
      for (int nd = 0; nd < nn; ++nd) {
        const int kb = __shfl_sync(0xffffffffu, ptr_l, nd), ke = __shfl_sync(0xffffffffu, ptr_l, nd + 1);
        if (ke - kb > HUB_DEG) {
          const long u0 = kb / HUB_UB;
          const int slot = __ldg(in_dst + u0 * HUB_UB) == int(t0 + nd) ? 0 : 1;
#pragma unroll
          for (int c = 0; c < V; ++c) acc[c] = hubsum[(u0 * 2 + slot) * D + lane * V + c];
        } else {
          for (int base = kb; base < ke; base += 32) {
            const int cnt = min(32, ke - base);
            const int sl = lane < cnt ? __ldg(in_src + base + lane) : 0;
            for (int j = 0; j < cnt; j += G) {
              RawRow<V, BF> gr[G], hr[G];
#pragma unroll
              for (int q = 0; q < G; ++q) {
                const int kk = min(j + q, cnt - 1);
                gr[q].load(g, long(base + kk), D, lane);
                hr[q].load(hbar, long(__shfl_sync(0xffffffffu, sl, kk)), D, lane);
              }
#pragma unroll
              for (int q = 0; q < G; ++q)
                if (j + q < cnt) {
                  float gv[V], hv[V];
                  gr[q].get(gv);
                  hr[q].get(hv);
#pragma unroll
                  for (int c = 0; c < V; ++c) acc[c] = fmaf(gv[c], hv[c], acc[c]);
                }
            }
          }
        }
        flush(nd);
      }
      node = nn;
    }
    for (int base = e_beg; base < e_end && !slow; base += 32) {
      const int cnt = min(32, e_end - base);
      if (base > e_beg) s_l = lane < cnt ? __ldg(in_src + base + lane) : 0;
      RawRow<V, BF> gr[G], hr[G], gn[G], hn[G];
      auto issue = [&](int j, RawRow<V, BF> (&ga)[G], RawRow<V, BF> (&ha)[G]) {
#pragma unroll
        for (int u = 0; u < G; ++u) {
          const int kk = min(j + u, cnt - 1);
          const int sidx = __shfl_sync(0xffffffffu, s_l, kk);
          ga[u].load(g, long(base + kk), D, lane);
          ha[u].load(hbar, long(sidx), D, lane);
        }
      };
      if (PF) issue(0, gn, hn);
      for (int j = 0; j < cnt; j += G) {
        if (PF) {
#pragma unroll
          for (int u = 0; u < G; ++u) {
            gr[u] = gn[u];
            hr[u] = hn[u];
          }
          if (j + G < cnt) issue(j + G, gn, hn);        // next round in flight while this one sums
        } else {
          issue(j, gr, hr);
        }
        if (!next_src_issued && t1 < N) {                      // next chunk's first sources
          const int nb = __shfl_sync(0xffffffffu, ptr_n, 0);
          const int n1 = int(min(long(NPW), N - t1));
          const int ne = __shfl_sync(0xffffffffu, ptr_n, n1);
          s_next = nb + lane < ne ? __ldg(in_src + nb + lane) : 0;
          next_src_issued = true;
        }
#pragma unroll
        for (int u = 0; u < G; ++u) {
          if (j + u < cnt) {
            const int k = base + j + u;
            while (k >= seg_end) {
              flush(node);
              ++node;
              seg_end = __shfl_sync(0xffffffffu, ptr_l, node + 1);
            }
            float gv[V], hv[V];
            gr[u].get(gv);
            hr[u].get(hv);
#pragma unroll
            for (int c = 0; c < V; ++c) acc[c] = fmaf(gv[c], hv[c], acc[c]);
          }
        }
      }
    }
    for (; node < nn; ++node) flush(node);
    if (!next_src_issued && t1 < N) {
      const int nb = __shfl_sync(0xffffffffu, ptr_n, 0);
      const int n1 = int(min(long(NPW), N - t1));
      const int ne = __shfl_sync(0xffffffffu, ptr_n, n1);
      s_next = nb + lane < ne ? __ldg(in_src + nb + lane) : 0;
    }
    ptr_l = ptr_n;
    s_first = s_next;
  }
}

// ---------------------------------------------------------------------------
// a10, gate / message backward with the forward's gates g (no recompute): per edge k,
//   dm = dA[t_k] (LReLU' and ÷deg already applied), MG = dm ⊙ g, dg = dm ⊙ h̄[s_k],
//   DV = g ⊙ (dg − ⟨g, dg⟩)          (softmax backward; ⟨·,·⟩ accumulated in float64)
// A warp takes 32 consecutive in-CSR edges, four at a time with all row loads of the
// four in flight; lane = D/32 channels; the dot is a fixed-order butterfly.
// ---------------------------------------------------------------------------
// MSGB (reading B, NEXT-1): g holds the per-channel in-edge softmax weights w; the segmented
// softmax backward dv_k = w_k ⊙ (dg_k - Σ_{k'∈seg(t)} w_k' ⊙ dg_k') with dg_k = dA_t ⊙ h̄[s_k]
// has Σ_{k'} w_k' ⊙ dg_k' = dA_t ⊙ A_t (A_t = Σ_k' w_k' ⊙ h̄[s_k'], the un-divided segment sum,
// recovered from h_t = LReLU(A_t / deg_t)), so dv_k = w_k ⊙ dA_t ⊙ (h̄[s_k] - A_t).
template <int D, bool BF, bool MSGB = false>
__global__ void __launch_bounds__(NT) gate_bwd_stream_kernel(
    const void *__restrict__ g, const float *__restrict__ dA, const void *__restrict__ hbar,
    const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst, int E,
    float *__restrict__ MG, float *__restrict__ DV, const float *__restrict__ h = nullptr,
    const int32_t *__restrict__ in_ptr = nullptr, int mean = 0, float slope = 0.01f,
    int *__restrict__ dv_rexp = nullptr) {
  // dv_rexp: the fp16x2 scale exponent of each DV row (max |DV| over the row), read by the
  // W_m row-GEMM's converters instead of a row-max pass of their own
  constexpr int V = D / 32;
  constexpr int G = 4;
  const int lane = threadIdx.x & 31;
  const long nwarps = long(gridDim.x) * (NT / 32);
  for (long k0 = (blockIdx.x * long(NT / 32) + threadIdx.x / 32) * 32; k0 < E; k0 += nwarps * 32) {
    const int cnt = int(min(32L, E - k0));
    const int s_l = lane < cnt ? __ldg(in_src + k0 + lane) : 0;
    const int t_l = lane < cnt ? __ldg(in_dst + k0 + lane) : 0;
    for (int j = 0; j < cnt; j += G) {
      RawRow<V, BF> gr[G], hr[G];
      RawRow<V, false> dr[G], ar[MSGB ? G : 1];
      float dsc[MSGB ? G : 1];
#pragma unroll
      for (int u = 0; u < G; ++u) {
        const int kk = min(j + u, cnt - 1);
        const int tk = __shfl_sync(0xffffffffu, t_l, kk);
        gr[u].load(g, k0 + kk, D, lane);
        dr[u].load(dA, tk, D, lane);
        hr[u].load(hbar, __shfl_sync(0xffffffffu, s_l, kk), D, lane);
        if constexpr (MSGB) {
          ar[u].load(h, tk, D, lane);
          dsc[u] = 1.f;
          if (mean) {
            const int deg = __ldg(in_ptr + tk + 1) - __ldg(in_ptr + tk);
            dsc[u] = float(deg > 0 ? deg : 1);
          }
        }
      }
#pragma unroll
      for (int u = 0; u < G; ++u) {
        if (j + u >= cnt) break;                       // warp-uniform
        float gv[V], dv[V], hv[V], dg[V];
        gr[u].get(gv);
        dr[u].get(dv);
        hr[u].get(hv);
        if constexpr (MSGB) {
          float av[V], mg[V], dvv[V];
          ar[u].get(av);
#pragma unroll
          for (int c = 0; c < V; ++c) {
            const float At = (av[c] > 0.f ? av[c] : av[c] / slope) * dsc[u];   // LReLU⁻¹, × deg
            mg[c] = dv[c] * gv[c];
            dvv[c] = mg[c] * (hv[c] - At);
          }
          if (MG) store_row<V>(MG + (k0 + j + u) * D + lane * V, mg);
          store_row<V>(DV + (k0 + j + u) * D + lane * V, dvv);
          continue;
        }
        double dot = 0.0;
#pragma unroll
        for (int c = 0; c < V; ++c) {
          dg[c] = dv[c] * hv[c];
          dot = fma(double(gv[c]), double(dg[c]), dot);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, o);
        const float dotf = float(dot);
        float mg[V], dvv[V];
#pragma unroll
        for (int c = 0; c < V; ++c) {
          mg[c] = dv[c] * gv[c];
          dvv[c] = gv[c] * (dg[c] - dotf);
        }
        if (MG) store_row<V>(MG + (k0 + j + u) * D + lane * V, mg);
        store_row<V>(DV + (k0 + j + u) * D + lane * V, dvv);
        if (dv_rexp) {        // row max |DV|: one warp integer max-reduce of the |x| bit patterns
          float mx = 0.f;
#pragma unroll
          for (int c = 0; c < V; ++c) mx = fmaxf(mx, fabsf(dvv[c]));
          mx = __uint_as_float(__reduce_max_sync(0xffffffffu, __float_as_uint(mx)));
          if (lane == 0) dv_rexp[k0 + j + u] = occu_row_scale_exp(mx);
        }
      }
    }
  }
}

// ---------------------------------------------------------------------------
// a4-a6 under reading B (NEXT-1; P149 with the softmax taken over the in-edges
// of the destination, per channel): with logits v_k = W_m e'_k (tensor-core plain GEMM),
//   w_kc = exp(v_kc - M_tc) / Σ_{k'∈seg(t)} exp(v_k'c - M_tc),   A_tc = Σ_{k∈seg(t)} w_kc h̄[s_k]c
// h_t = LReLU(A_t) (÷ deg for MEAN; an empty segment gives 0).  One pass per segment with an
// online maximum and rescaled running sums per lane-channel, edges in ascending in-CSR order
// (fixed order, atomic-free).  Warps walk chunks of 8 destinations; G (v, h̄[s]) row pairs of
// the chunk are in flight at a time.  W (training): a second pass over each finished segment
// overwrites v_k with w_k (the weights the backward reads; each row is read before it is
// written and only by its owner warp).  RP: last layer, readout chunk partials as v2.
// ---------------------------------------------------------------------------
// BF (OCCU_BF16): v, h̄ and h are BF16 rows (the softmax, the sums and the readout stay FP32).
template <int D, int G, bool RP, bool W, bool BF>
__global__ void __launch_bounds__(NT) gather_segsoftmax_kernel(
    void *__restrict__ v, const void *__restrict__ hbar, const int32_t *__restrict__ in_ptr,
    const int32_t *__restrict__ in_src, int N, int mean, float slope, void *__restrict__ h_out,
    const int32_t *__restrict__ node_graph, float *__restrict__ rpart) {
  constexpr int V = D / 32;
  constexpr int NPW = 8;
  constexpr float L2E = 1.4426950408889634f;
  const int lane = threadIdx.x & 31;
  const long nw = (long(gridDim.x) * NT) / 32;
  pdl_trigger();
  pdl_wait();
  for (long t0 = (blockIdx.x * long(NT) + threadIdx.x) / 32 * NPW; t0 < N; t0 += nw * NPW) {
    const int nn = int(min(long(NPW), N - t0));
    const int ptr_l = lane <= nn ? __ldg(in_ptr + t0 + lane) : 0;
    const int gr_l = (RP && lane < nn) ? __ldg(node_graph + t0 + lane) : -1;
    const int e_beg = __shfl_sync(0xffffffffu, ptr_l, 0);
    const int e_end = __shfl_sync(0xffffffffu, ptr_l, nn);
    int node = 0;
    int seg_beg = e_beg;
    int seg_end = __shfl_sync(0xffffffffu, ptr_l, 1);
    float m[V], sum[V], acc[V], racc[V];
#pragma unroll
    for (int c = 0; c < V; ++c) {
      m[c] = -INFINITY;
      sum[c] = acc[c] = racc[c] = 0.f;
    }
    auto flush = [&](int nd) {
      const int deg = seg_end - seg_beg;
      float o[V];
#pragma unroll
      for (int c = 0; c < V; ++c) {
        float x = deg > 0 ? acc[c] / sum[c] : 0.f;
        if (mean) x = x / float(deg > 0 ? deg : 1);
        o[c] = lrelu(x, slope);
      }
      if (W && deg > 0) {                   // weights of the finished segment, in place
        float inv[V];
#pragma unroll
        for (int c = 0; c < V; ++c) inv[c] = 1.f / sum[c];
        for (int k = seg_beg; k < seg_end; ++k) {
          float x[V];
          load_row<V, BF>(v, long(k), D, lane, x);
#pragma unroll
          for (int c = 0; c < V; ++c) x[c] = ex2f_fast((x[c] - m[c]) * L2E) * inv[c];
          store_row_t<V, BF>(v, long(k), D, lane, x);
        }
      }
#pragma unroll
      for (int c = 0; c < V; ++c) {
        m[c] = -INFINITY;
        sum[c] = acc[c] = 0.f;
      }
      if (!RP || h_out) store_row_t<V, BF>(h_out, t0 + nd, D, lane, o);
      if (RP) {
        const int gc = __shfl_sync(0xffffffffu, gr_l, nd);
        const int gn = __shfl_sync(0xffffffffu, gr_l, (nd + 1) & 31);
#pragma unroll
        for (int c = 0; c < V; ++c) racc[c] += o[c];
        if (nd + 1 >= nn || gn != gc) {
          store_row<V>(rpart + (t0 + nd) * D + lane * V, racc);
#pragma unroll
          for (int c = 0; c < V; ++c) racc[c] = 0.f;
        }
      }
    };
    for (int base = e_beg; base < e_end; base += 32) {
      const int cnt = min(32, e_end - base);
      const int s_l = lane < cnt ? __ldg(in_src + base + lane) : 0;
      for (int j = 0; j < cnt; j += G) {
        RawRow<V, BF> vr[G], hr[G];
#pragma unroll
        for (int u = 0; u < G; ++u) {
          const int kk = min(j + u, cnt - 1);
          vr[u].load(v, long(base + kk), D, lane);
          hr[u].load(hbar, long(__shfl_sync(0xffffffffu, s_l, kk)), D, lane);
        }
#pragma unroll
        for (int u = 0; u < G; ++u) {
          if (j + u < cnt) {
            const int k = base + j + u;
            while (k >= seg_end) {
              flush(node);
              ++node;
              seg_beg = seg_end;
              seg_end = __shfl_sync(0xffffffffu, ptr_l, node + 1);
            }
            float xv[V], hv[V];
            vr[u].get(xv);
            hr[u].get(hv);
#pragma unroll
            for (int c = 0; c < V; ++c) {
              if (xv[c] > m[c]) {            // new maximum: rescale the running sums
                const float sc = ex2f_fast((m[c] - xv[c]) * L2E);
                sum[c] = fmaf(sum[c], sc, 1.f);
                acc[c] = fmaf(acc[c], sc, hv[c]);
                m[c] = xv[c];
              } else {
                const float e = ex2f_fast((xv[c] - m[c]) * L2E);
                sum[c] += e;
                acc[c] = fmaf(e, hv[c], acc[c]);
              }
            }
          }
        }
      }
    }
    for (; node < nn; ++node) {
      flush(node);
      seg_beg = seg_end;
      seg_end = __shfl_sync(0xffffffffu, ptr_l, min(node + 2, nn));
    }
  }
}

// cp.async helpers of the per-warp shared-memory row rings (edge / node backward)
template <int N>
__device__ __forceinline__ void cpa_ca(void *dst, const void *src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(dst))),
               "l"(src), "n"(N) : "memory");
}
__device__ __forceinline__ void cpa_commit_nb() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cpa_wait_nb() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// ---------------------------------------------------------------------------
// a10, layer-1 edge backward (F_e = Ke <= KM small; the edge transform was a CUDA-core step):
//   z = W_e e0_k (recomputed from the saved permuted features), y = α z,
//   dy = de ⊙ e' ⊙ σ(-y), dα = <dy, z> (float64), DZ = α dy.
// A warp takes 32 consecutive in-CSR edges: lane j loads edge j's α and Ke features (all in
// flight), then the warp walks the edges four at a time with the e' / de rows of the four in
// flight; lane = D/32 channels (coalesced rows), W_e's columns for the lane's channels live in
// registers; the dot is a fixed-order butterfly.  BF: e' rows are BF16 (OCCU_BF16 training).
// FUSEW (KM = Ke = 4): the layer's weight gradient dW_e = DZᵀ e0 is accumulated here as well
// (lane = its channels x the Ke features, FP32 over the warp's edges, warps combined in fixed
// order per block) into per-block partials dwe_part[block][D][Ke], reduced in block order by
// the layer's multi_reduce — DZ is not read back by a weight-gradient kernel.
// ---------------------------------------------------------------------------
// CPA: the edge's e' and de rows land by cp.async in a per-warp shared-memory ring of EB_RING
// slots instead of G register rows (the same rows in the same order: bitwise equal)
#ifndef OCCU_EB_RING
#define OCCU_EB_RING 6
#endif
constexpr int EB_RING = OCCU_EB_RING;
template <int D, bool BF> constexpr int eb_slot_bytes() { return D * (BF ? 2 : 4) + D * 4; }
template <int D, int KM, bool BF, bool FUSEW = false, bool CPA = false>
__global__ void __launch_bounds__(NT, CPA ? 3 : 1) edge_bwd_small_kernel(
    const float *__restrict__ e0, int Ke, const void *__restrict__ e, const float *__restrict__ de,
    const float *__restrict__ W_e, const float *__restrict__ p, const float *__restrict__ q,
    const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst, int E,
    float *__restrict__ DZ, float *__restrict__ dalpha, float *__restrict__ dwe_part = nullptr) {
  static_assert(!FUSEW || KM == 4, "fused dW_e: Ke = 4 only");
  constexpr int V = D / 32;
  constexpr int G = 4;
  constexpr float L2E = 1.4426950408889634f;
  const int lane = threadIdx.x & 31;
  float w[KM][V];
#pragma unroll
  for (int j = 0; j < KM; ++j)
#pragma unroll
    for (int c = 0; c < V; ++c) w[j][c] = j < Ke ? __ldg(W_e + long(lane * V + c) * Ke + j) : 0.f;
  float gw[FUSEW ? V : 1][FUSEW ? KM : 1];
#pragma unroll
  for (int c = 0; c < (FUSEW ? V : 1); ++c)
#pragma unroll
    for (int j = 0; j < (FUSEW ? KM : 1); ++j) gw[c][j] = 0.f;
  const long nwarps = long(gridDim.x) * (NT / 32);
  for (long k0 = (blockIdx.x * long(NT / 32) + threadIdx.x / 32) * 32; k0 < E; k0 += nwarps * 32) {
    const int cnt = int(min(32L, E - k0));
    float al = 0.f, ev[KM];
#pragma unroll
    for (int j = 0; j < KM; ++j) ev[j] = 0.f;
    if (lane < cnt) {
      const long k = k0 + lane;
      al = __ldg(p + __ldg(in_src + k)) + __ldg(q + __ldg(in_dst + k));
      if (KM == 4 && Ke == 4) {
        const float4 x = __ldg(reinterpret_cast<const float4 *>(e0 + k * 4));
        ev[0] = x.x; ev[1 % KM] = x.y; ev[2 % KM] = x.z; ev[3 % KM] = x.w;
      } else {
#pragma unroll
        for (int j = 0; j < KM; ++j) ev[j] = j < Ke ? __ldg(e0 + k * Ke + j) : 0.f;
      }
    }
    float dal_mine = 0.f;
    auto process = [&](int kk, const float (&evv)[V], const float (&dvv)[V]) {
      const float a = __shfl_sync(0xffffffffu, al, kk);
      float z[V], xs[KM];
#pragma unroll
      for (int c = 0; c < V; ++c) z[c] = 0.f;
#pragma unroll
      for (int j = 0; j < KM; ++j) {
        const float x = __shfl_sync(0xffffffffu, ev[j], kk);
        xs[j] = x;
#pragma unroll
        for (int c = 0; c < V; ++c) z[c] = fmaf(w[j][c], x, z[c]);
      }
      float o[V];
      double dot = 0.0;
#pragma unroll
      for (int c = 0; c < V; ++c) {
        // σ'(y) = σ(y)·σ(-y) with σ(y) = e' (stored) and y = α z recomputed
        const float dy = dvv[c] * evv[c] * __frcp_rn(1.f + ex2f_fast(a * z[c] * L2E));
        dot = fma(double(dy), double(z[c]), dot);
        o[c] = a * dy;
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, off);
      store_row<V>(DZ + (k0 + kk) * D + lane * V, o);
      if (lane == kk) dal_mine = float(dot);
      if constexpr (FUSEW) {
#pragma unroll
        for (int c = 0; c < V; ++c)
#pragma unroll
          for (int j = 0; j < KM; ++j) gw[c][j] = fmaf(o[c], xs[j], gw[c][j]);    // DZᵀ e0, edge order
      }
    };
    if constexpr (CPA) {
      extern __shared__ __align__(16) uint8_t eb_dyn[];
      constexpr int EB = BF ? 2 : 4, SLOT = eb_slot_bytes<D, BF>();
      uint8_t *ring = eb_dyn + (threadIdx.x / 32) * (EB_RING * SLOT);
      auto issue1 = [&](int jj) {                     // edge jj of the batch -> slot jj % EB_RING
        if (jj < cnt) {
          uint8_t *sp = ring + (jj % EB_RING) * SLOT;
          cpa_ca<V * EB>(sp + lane * V * EB, reinterpret_cast<const uint8_t *>(e) + ((k0 + jj) * D + lane * V) * EB);
          cpa_ca<V * 4>(sp + D * EB + lane * V * 4, de + (k0 + jj) * D + lane * V);
        }
        cpa_commit_nb();
      };
#pragma unroll
      for (int q = 0; q < EB_RING; ++q) issue1(q);
      for (int kk = 0; kk < cnt; ++kk) {
        cpa_wait_nb<EB_RING - 1>();
        const uint8_t *sp = ring + (kk % EB_RING) * SLOT;
        float evv[V], dvv[V];
#pragma unroll
        for (int c = 0; c < V; ++c) {
          evv[c] = BF ? __uint_as_float(uint32_t(reinterpret_cast<const uint16_t *>(sp)[lane * V + c]) << 16)
                      : reinterpret_cast<const float *>(sp)[lane * V + c];
          dvv[c] = reinterpret_cast<const float *>(sp + D * EB)[lane * V + c];
        }
        process(kk, evv, dvv);
        issue1(kk + EB_RING);
      }
      cpa_wait_nb<0>();
    } else {
      for (int jb = 0; jb < cnt; jb += G) {
        RawRow<V, BF> er[G];
        RawRow<V, false> dr[G];
#pragma unroll
        for (int u = 0; u < G; ++u) {
          const int kk = min(jb + u, cnt - 1);
          er[u].load(e, k0 + kk, D, lane);
          dr[u].load(de, k0 + kk, D, lane);
        }
#pragma unroll
        for (int u = 0; u < G; ++u) {
          if (jb + u >= cnt) break;                     // warp-uniform
          float evv[V], dvv[V];
          er[u].get(evv);
          dr[u].get(dvv);
          process(jb + u, evv, dvv);
        }
      }
    }
    if (lane < cnt) dalpha[k0 + lane] = dal_mine;
  }
  if constexpr (FUSEW) {
    __shared__ float red[NT / 32][D * KM];
    const int wl = threadIdx.x / 32;
#pragma unroll
    for (int c = 0; c < V; ++c)
#pragma unroll
      for (int j = 0; j < KM; ++j) red[wl][(lane * V + c) * KM + j] = gw[c][j];
    __syncthreads();
    for (int o = threadIdx.x; o < D * KM; o += NT) {
      double acc = 0.0;
      for (int w2 = 0; w2 < NT / 32; ++w2) acc += red[w2][o];
      dwe_part[long(blockIdx.x) * D * KM + o] = float(acc);
    }
  }
}

// e0[k] = edge_feat[in_eid[k]]  (a1)
__global__ void permute_rows_kernel(const float *__restrict__ src, const int32_t *__restrict__ idx,
                                    int rows, int width, float *__restrict__ dst) {
  const long total = long(rows) * width;
  for (long i = blockIdx.x * long(blockDim.x) + threadIdx.x; i < total;
       i += long(gridDim.x) * blockDim.x) {
    const long r = i / width, c = i % width;
    dst[i] = src[long(idx[r]) * width + c];
  }
}

// ---------------------------------------------------------------------------
// a7 + a8: readout (mean over the graph's nodes) and head, one CTA of 16 warps per
// graph.  Warp w sums rows w, w+16, ... (lane = D/32 channels, 4 rows in flight);
// the 16 warp partials are combined in fixed order.  chunk == 0: the rows are the
// node states h_u; chunk > 0: they are gather_segsum_kernel's chunk partials (graph
// b's rows are min(u1 - 1, chunk*c + chunk - 1), c = u0/chunk .. (u1-1)/chunk).
// Head: warp per hidden unit j (lanes over k, coalesced W_1 rows), butterfly sums.
// ---------------------------------------------------------------------------
constexpr int RO_WARPS = 16;
template <int D>
__global__ void __launch_bounds__(RO_WARPS * 32) readout_head_kernel(
    const float *__restrict__ h, const int32_t *__restrict__ node_off, int d_h,
    const float *__restrict__ W_1, const float *__restrict__ b_1, const float *__restrict__ w_2,
    const float *__restrict__ b_2, float slope, float *__restrict__ r_out,
    float *__restrict__ c_out, float *__restrict__ yhat, int chunk) {
  constexpr int V = D / 32;
  extern __shared__ float sm[];
  pdl_trigger();
  pdl_wait();
  float *part = sm;                    // [RO_WARPS][D]
  float *rs = part + RO_WARPS * D;     // [D]
  float *os = rs + D;                  // [d_h]
  const int b = blockIdx.x;
  const int u0 = node_off[b], u1 = node_off[b + 1];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int k0 = chunk > 0 ? u0 / chunk : u0, k1 = chunk > 0 ? (u1 - 1) / chunk + 1 : u1;
  float acc[V];
#pragma unroll
  for (int c = 0; c < V; ++c) acc[c] = 0.f;
  auto row_of = [&](int k) { return chunk > 0 ? min(u1 - 1, k * chunk + chunk - 1) : k; };
  int k = k0 + warp;
  for (; k + 3 * RO_WARPS < k1; k += 4 * RO_WARPS) {
    float x[4][V];
#pragma unroll
    for (int t = 0; t < 4; ++t) load_row<V, false>(h, long(row_of(k + t * RO_WARPS)), D, lane, x[t]);
#pragma unroll
    for (int t = 0; t < 4; ++t)
#pragma unroll
      for (int c = 0; c < V; ++c) acc[c] += x[t][c];
  }
  for (; k < k1; k += RO_WARPS) {
    float x[V];
    load_row<V, false>(h, long(row_of(k)), D, lane, x);
#pragma unroll
    for (int c = 0; c < V; ++c) acc[c] += x[c];
  }
#pragma unroll
  for (int c = 0; c < V; ++c) part[warp * D + lane * V + c] = acc[c];
  __syncthreads();
  if (threadIdx.x < D) {
    float sum = 0.f;
#pragma unroll
    for (int w = 0; w < RO_WARPS; ++w) sum += part[w * D + threadIdx.x];
    const float rv = sum / float(u1 - u0);
    rs[threadIdx.x] = rv;
    r_out[long(b) * D + threadIdx.x] = rv;
  }
  __syncthreads();
  for (int j0 = warp; j0 < d_h; j0 += 4 * RO_WARPS) {
    float cv[4];
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      const int j = j0 + t * RO_WARPS;
      cv[t] = 0.f;
      if (j < d_h) {
        float w[V];
        load_row<V, false>(W_1, long(j), D, lane, w);     // coalesced vector loads of row j
#pragma unroll
        for (int c = 0; c < V; ++c) cv[t] = fmaf(w[c], rs[lane * V + c], cv[t]);
      }
    }
#pragma unroll
    for (int t = 0; t < 4; ++t) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) cv[t] += __shfl_xor_sync(0xffffffffu, cv[t], o);
      const int j = j0 + t * RO_WARPS;
      if (lane == 0 && j < d_h) {
        const float v = cv[t] + b_1[j];
        c_out[long(b) * d_h + j] = v;
        os[j] = lrelu(v, slope);
      }
    }
  }
  __syncthreads();
  if (warp == 0) {
    float y = 0.f;
    for (int j = lane; j < d_h; j += 32) y = fmaf(__ldg(w_2 + j), os[j], y);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) y += __shfl_xor_sync(0xffffffffu, y, o);
    if (lane == 0) yhat[b] = y + b_2[0];
  }
}

// ---------------------------------------------------------------------------
// Backward.
// ---------------------------------------------------------------------------
// Per graph: dŷ_b = 2(ŷ_b - y_b)/B_glob ; dc = dŷ w_2 ⊙ LReLU'(c) ; dr = W_1ᵀ dc
__global__ void head_bwd_graph_kernel(const float *__restrict__ yhat, const float *__restrict__ y,
                                      const float *__restrict__ c, const float *__restrict__ W_1,
                                      const float *__restrict__ w_2, int D, int d_h, float inv_gb,
                                      float slope, float *__restrict__ dy, float *__restrict__ dc,
                                      float *__restrict__ dr) {
  extern __shared__ float sm[];
  const int b = blockIdx.x;
  const float d = 2.f * (yhat[b] - y[b]) * inv_gb;
  for (int j = threadIdx.x; j < d_h; j += blockDim.x) {
    const float cv = c[long(b) * d_h + j];
    const float v = d * w_2[j] * (cv > 0.f ? 1.f : slope);
    sm[j] = v;
    dc[long(b) * d_h + j] = v;
  }
  if (threadIdx.x == 0) dy[b] = d;
  __syncthreads();
  for (int k = threadIdx.x; k < D; k += blockDim.x) {
    float s = 0.f;
    for (int j = 0; j < d_h; ++j) s = fmaf(W_1[long(j) * D + k], sm[j], s);
    dr[long(b) * D + k] = s;
  }
}

// Head parameter gradients and the loss, each a fixed-order sum over graphs.
__global__ void head_bwd_reduce_kernel(const float *__restrict__ dy, const float *__restrict__ dc,
                                       const float *__restrict__ r, const float *__restrict__ c,
                                       const float *__restrict__ yhat, const float *__restrict__ y,
                                       int B, int D, int d_h, float inv_gb, float slope,
                                       float *__restrict__ gW_1, float *__restrict__ gb_1,
                                       float *__restrict__ gw_2, float *__restrict__ gb_2,
                                       float *__restrict__ loss) {
  const int jobs = d_h * D + 2 * d_h + 2;
  for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < jobs; t += gridDim.x * blockDim.x) {
    float s = 0.f;
    if (t < d_h * D) {
      const int j = t / D, k = t % D;
      for (int b = 0; b < B; ++b) s = fmaf(dc[long(b) * d_h + j], r[long(b) * D + k], s);
      gW_1[t] = s;
    } else if (t < d_h * D + d_h) {
      const int j = t - d_h * D;
      for (int b = 0; b < B; ++b) s += dc[long(b) * d_h + j];
      gb_1[j] = s;
    } else if (t < d_h * D + 2 * d_h) {
      const int j = t - d_h * D - d_h;
      for (int b = 0; b < B; ++b) s = fmaf(dy[b], lrelu(c[long(b) * d_h + j], slope), s);
      gw_2[j] = s;
    } else if (t == d_h * D + 2 * d_h) {
      for (int b = 0; b < B; ++b) s += dy[b];
      gb_2[0] = s;
    } else {
      for (int b = 0; b < B; ++b) {
        const float e = yhat[b] - y[b];
        s = fmaf(e, e, s);
      }
      loss[0] = s * inv_gb;
    }
  }
}

// dh^L_u = dr_{graph(u)} / n_{graph(u)}
// h_mask != null: emit dA = dh ⊙ LReLU'(A) (÷ deg for MEAN; sign(A) = sign(h)) instead of dh.
// Thread = (node, 4 consecutive channels): float4 loads / stores, one node_graph lookup.
// The d = 128 sign-bit case of broadcast_dh_kernel with more loads in flight: warp = 4 nodes
// per step, lane = 4 channels; each dependent load level (node_graph -> node_off / dr row / mask
// word) is issued for all 4 nodes before any is used.  Same arithmetic per element (bitwise).
__global__ void __launch_bounds__(256) broadcast_dh_bits128_kernel(
    const float *__restrict__ dr, const int32_t *__restrict__ node_graph,
    const int32_t *__restrict__ node_off, int N, const int32_t *__restrict__ in_ptr, int mean,
    float slope, float *__restrict__ dh, const uint32_t *__restrict__ h_bits) {
  constexpr int D = 128, Q = 4;
  const int lane = threadIdx.x & 31;
  const long nw = long(gridDim.x) * (blockDim.x / 32);
  for (long u0 = (long(blockIdx.x) * (blockDim.x / 32) + threadIdx.x / 32) * Q; u0 < N; u0 += nw * Q) {
    int b[Q];
    uint4 w[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const long u = u0 + q;
      b[q] = u < N ? __ldg(node_graph + u) : 0;
      w[q] = u < N ? __ldg(reinterpret_cast<const uint4 *>(h_bits) + u) : make_uint4(0u, 0u, 0u, 0u);
    }
    float inv[Q], dsc[Q];
    float4 r[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const long u = u0 + q;
      inv[q] = 1.f / float(__ldg(node_off + b[q] + 1) - __ldg(node_off + b[q]));
      r[q] = __ldg(reinterpret_cast<const float4 *>(dr + long(b[q]) * D) + lane);
      dsc[q] = 1.f;
      if (mean && u < N) {
        const int deg = __ldg(in_ptr + u + 1) - __ldg(in_ptr + u);
        dsc[q] = float(deg > 0 ? deg : 1);
      }
    }
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const long u = u0 + q;
      if (u >= N) break;
      float v[4] = {r[q].x * inv[q], r[q].y * inv[q], r[q].z * inv[q], r[q].w * inv[q]};
      const uint32_t wc[4] = {w[q].x, w[q].y, w[q].z, w[q].w};
#pragma unroll
      for (int c = 0; c < 4; ++c) {                   // channel 4·lane + c: word c, bit lane
        v[c] = v[c] * lrelu_grad_from_out((wc[c] >> lane) & 1u ? 1.f : -1.f, slope);
        if (mean) v[c] = v[c] / dsc[q];
      }
      reinterpret_cast<float4 *>(dh + u * D)[lane] = make_float4(v[0], v[1], v[2], v[3]);
    }
  }
}

__global__ void broadcast_dh_kernel(const float *__restrict__ dr, const int32_t *__restrict__ node_graph,
                                    const int32_t *__restrict__ node_off, int N, int D,
                                    const void *__restrict__ h_mask, int mask_bf,
                                    const int32_t *__restrict__ in_ptr,
                                    int mean, float slope, float *__restrict__ dh,
                                    const uint32_t *__restrict__ h_bits) {
  // h_bits (training forward's sign bits of h_L, word c / bit l = channel V·l + c) replace the
  // h_L rows as the LReLU' mask: D/8 bytes per node instead of a D-wide row
  const int D4 = D / 4;
  const long total = long(N) * D4;
  for (long i = blockIdx.x * long(blockDim.x) + threadIdx.x; i < total;
       i += long(gridDim.x) * blockDim.x) {
    const int u = int(i / D4), k4 = int(i % D4);
    const int b = __ldg(node_graph + u);
    const float inv = 1.f / float(__ldg(node_off + b + 1) - __ldg(node_off + b));
    const float4 r = __ldg(reinterpret_cast<const float4 *>(dr + long(b) * D) + k4);
    float v[4] = {r.x * inv, r.y * inv, r.z * inv, r.w * inv};
    if (h_bits || h_mask) {
      float hm[4];
      if (h_bits && D == 128) {        // channel 4·k4 + c: word c, bit k4
        const uint4 w = __ldg(reinterpret_cast<const uint4 *>(h_bits) + u);
        hm[0] = (w.x >> k4) & 1u ? 1.f : -1.f;
        hm[1] = (w.y >> k4) & 1u ? 1.f : -1.f;
        hm[2] = (w.z >> k4) & 1u ? 1.f : -1.f;
        hm[3] = (w.w >> k4) & 1u ? 1.f : -1.f;
      } else if (h_bits) {
        const int V = D / 32;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const int ch = 4 * k4 + c;
          hm[c] = (__ldg(h_bits + long(u) * V + ch % V) >> (ch / V)) & 1u ? 1.f : -1.f;
        }
      } else if (mask_bf) {
        const uint2 x = __ldg(reinterpret_cast<const uint2 *>(reinterpret_cast<const uint16_t *>(h_mask) + long(u) * D) + k4);
        hm[0] = __uint_as_float(x.x << 16); hm[1] = __uint_as_float(x.x & 0xFFFF0000u);
        hm[2] = __uint_as_float(x.y << 16); hm[3] = __uint_as_float(x.y & 0xFFFF0000u);
      } else {
        const float4 x = __ldg(reinterpret_cast<const float4 *>(reinterpret_cast<const float *>(h_mask) + long(u) * D) + k4);
        hm[0] = x.x; hm[1] = x.y; hm[2] = x.z; hm[3] = x.w;
      }
      float dsc = 1.f;
      if (mean) {
        const int deg = __ldg(in_ptr + u + 1) - __ldg(in_ptr + u);
        dsc = float(deg > 0 ? deg : 1);
      }
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        v[c] = v[c] * lrelu_grad_from_out(hm[c], slope);
        if (mean) v[c] = v[c] / dsc;
      }
    }
    reinterpret_cast<float4 *>(dh + long(u) * D)[k4] = make_float4(v[0], v[1], v[2], v[3]);
  }
}

// Edge backward, phase A (W_m): recompute g = softmax(W_m e'), then
//   dm = dA[t] ; dg = dm ⊙ h̄[s] ; MG = dm ⊙ g ; dv = g ⊙ (dg - <g,dg>) ;
//   de = W_mᵀ dv + de_out.
// dA[t] = dh[t] ⊙ LReLU'(A_t) (÷ deg for MEAN); sign(A) = sign(h).
template <int D>
__global__ void __launch_bounds__(NT) edge_bwd_m_kernel(
    const float *__restrict__ e, const float *__restrict__ W_m, const float *__restrict__ hbar,
    const float *__restrict__ h, const float *__restrict__ dh, const float *__restrict__ de_out,
    const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst,
    const int32_t *__restrict__ in_ptr, int E, int mean, float slope,
    float *__restrict__ MG, float *__restrict__ DV, float *__restrict__ de) {
  extern __shared__ __align__(16) float smem[];
  float *WmT = smem;               // [D][D] W_mᵀ
  float *Wm = WmT + D * D;         // [D][D] W_m
  float *As = Wm + D * D;          // [BM][D+4]
  int *sidx = reinterpret_cast<int *>(As + BM * (D + 4));   // [BM] src
  int *tidx = sidx + BM;                                      // [BM] dst
  constexpr int TN = Tn<D>::v;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  load_weights<D, true>(WmT, W_m, D);
  load_weights<D, false>(Wm, W_m, D);
  const int tiles = (E + BM - 1) / BM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long k0 = long(tile) * BM;
    const int nrows = min(BM, int(E - k0));
    __syncthreads();
    load_rows(As, e, k0, nrows, D);
    if (threadIdx.x < BM) {
      const int r = threadIdx.x;
      sidx[r] = r < nrows ? in_src[k0 + r] : 0;
      tidx[r] = r < nrows ? in_dst[k0 + r] : 0;
    }
    __syncthreads();
    float acc[4][TN];
    zero_acc<D>(acc);
    gemm_tile<D>(As, D, WmT, acc, tx, ty);
    float dv[4][TN];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = ty * 4 + i;
      float mx = -INFINITY;
#pragma unroll
      for (int j = 0; j < TN; ++j) mx = fmaxf(mx, acc[i][j]);
      mx = hmax16(mx);
      float gg[TN], s = 0.f;
#pragma unroll
      for (int j = 0; j < TN; ++j) {
        gg[j] = expf(acc[i][j] - mx);
        s += gg[j];
      }
      s = hsum16(s);
#pragma unroll
      for (int j = 0; j < TN; ++j) gg[j] = gg[j] / s;
      const int t = tidx[r], sr = sidx[r];
      float dhv[TN], hv[TN], hb[TN];
      load_row<D>(dh + long(t) * D, dhv, tx);
      load_row<D>(h + long(t) * D, hv, tx);
      load_row<D>(hbar + long(sr) * D, hb, tx);
      float inv = 1.f;
      if (mean) {
        const int deg = in_ptr[t + 1] - in_ptr[t];
        inv = float(deg > 0 ? deg : 1);
      }
      float mg[TN], dg[TN];
      double dotd = 0.0;
#pragma unroll
      for (int j = 0; j < TN; ++j) {
        float dm = dhv[j] * lrelu_grad_from_out(hv[j], slope);
        if (mean) dm = dm / inv;
        dg[j] = dm * hb[j];
        mg[j] = dm * gg[j];
        dotd = fma(double(gg[j]), double(dg[j]), dotd);
      }
      const float dot = float(hsum16d(dotd));
#pragma unroll
      for (int j = 0; j < TN; ++j) dv[i][j] = gg[j] * (dg[j] - dot);
      if (r < nrows) {
        store_row<D>(MG + (k0 + r) * D, mg, tx);
        store_row<D>(DV + (k0 + r) * D, dv[i], tx);
      }
    }
    __syncthreads();   // everyone done reading As (e') -> reuse for dv
#pragma unroll
    for (int i = 0; i < 4; ++i) store_row<D>(As + (ty * 4 + i) * (D + 4), dv[i], tx);
    __syncthreads();
    zero_acc<D>(acc);
    gemm_tile<D>(As, D, Wm, acc, tx, ty);                    // W_mᵀ dv (row form dv W_m)
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = ty * 4 + i;
      if (r >= nrows) continue;
      float v[TN];
      if (de_out) {
        float o[TN];
        load_row<D>(de_out + (k0 + r) * D, o, tx);
#pragma unroll
        for (int j = 0; j < TN; ++j) v[j] = acc[i][j] + o[j];
      } else {
#pragma unroll
        for (int j = 0; j < TN; ++j) v[j] = acc[i][j];
      }
      store_row<D>(de + (k0 + r) * D, v, tx);
    }
  }
}

// Edge backward, phase B (W_e): dy = de ⊙ e'(1-e') ; z = W_e e_in (recompute) ;
// dα = <dy, z> ; dz = α dy ; de_prev = W_eᵀ dz (layer > 0).
template <int D, bool BF>
__global__ void __launch_bounds__(NT) edge_bwd_e_kernel(
    const float *__restrict__ e_in, int Ke, const void *__restrict__ e, const float *__restrict__ de,
    const float *__restrict__ W_e, const float *__restrict__ p, const float *__restrict__ q,
    const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst, int E,
    float *__restrict__ DZ, float *__restrict__ dalpha, float *__restrict__ de_prev) {
  extern __shared__ __align__(16) float smem[];
  float *WeT = smem;                 // [Ke][D]  W_eᵀ
  float *We = WeT + Ke * D;          // [D][Ke]  W_e (only when de_prev)
  float *As = We + (de_prev ? D * Ke : 0);    // [BM][max(Ke,D)+4]
  const int KS = (Ke > D ? Ke : D);
  float *alpha = As + BM * (KS + 4);
  constexpr int TN = Tn<D>::v;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  load_weights<D, true>(WeT, W_e, Ke);
  if (de_prev) {   // de_prev only when Ke == D; Ws[a][c'] = W_e[a][c']
    load_weights<D, false>(We, W_e, D);
  }
  const int tiles = (E + BM - 1) / BM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long k0 = long(tile) * BM;
    const int nrows = min(BM, int(E - k0));
    __syncthreads();
    load_rows(As, e_in, k0, nrows, Ke);
    if (threadIdx.x < BM) {
      const int r = threadIdx.x;
      alpha[r] = r < nrows ? p[in_src[k0 + r]] + q[in_dst[k0 + r]] : 0.f;
    }
    __syncthreads();
    float acc[4][TN];
    zero_acc<D>(acc);
    gemm_tile<D>(As, Ke, WeT, acc, tx, ty);                  // z
    float dz[4][TN];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = ty * 4 + i;
      float ev[TN], dev[TN];
      double dad = 0.0;
      if (r < nrows) {
        if constexpr (BF) {
#pragma unroll
          for (int j = 0; j < TN; ++j) ev[j] = ld_act<true>(e, (k0 + r) * D + colof<D>(tx, j));
        } else {
          load_row<D>(reinterpret_cast<const float *>(e) + (k0 + r) * D, ev, tx);
        }
        load_row<D>(de + (k0 + r) * D, dev, tx);
      } else {
#pragma unroll
        for (int j = 0; j < TN; ++j) ev[j] = dev[j] = 0.f;
      }
      const float al = alpha[r];
#pragma unroll
      for (int j = 0; j < TN; ++j) {
        // σ'(y) = σ(y)·σ(-y) with y = α z recomputed: avoids the cancellation of
        // 1 - e' when e' = σ(y) is close to 1 (float32).
        const float dyv = dev[j] * ev[j] * (1.f / (1.f + expf(al * acc[i][j])));
        dad = fma(double(dyv), double(acc[i][j]), dad);
        dz[i][j] = al * dyv;
      }
      const float da = float(hsum16d(dad));
      if (r < nrows) {
        store_row<D>(DZ + (k0 + r) * D, dz[i], tx);
        if (tx == 0) dalpha[k0 + r] = da;
      }
    }
    if (de_prev) {
      __syncthreads();
#pragma unroll
      for (int i = 0; i < 4; ++i) store_row<D>(As + (ty * 4 + i) * (D + 4), dz[i], tx);
      __syncthreads();
      zero_acc<D>(acc);
      gemm_tile<D>(As, D, We, acc, tx, ty);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int r = ty * 4 + i;
        if (r < nrows) store_row<D>(de_prev + (k0 + r) * D, acc[i], tx);
      }
    }
  }
}

// Node backward (warp per node u):
//   dh̄_u = Σ_{out-edges} MG + dp_u a_s + dq_u a_d ; dP = dh̄ ⊙ LReLU'(h̄)
//   dp_u = Σ_{out-edges} dα ; dq_u = Σ_{in-edges} dα
template <int D, bool BF>
__global__ void __launch_bounds__(NT) node_bwd_kernel(
    const float *__restrict__ MG, const float *__restrict__ dalpha,
    const void *__restrict__ hbar, const float *__restrict__ a_s, const float *__restrict__ a_d,
    const int32_t *__restrict__ out_ptr, const int32_t *__restrict__ out_pos,
    const int32_t *__restrict__ in_ptr, int N, float slope, float *__restrict__ dP,
    float *__restrict__ dpq, float *__restrict__ da_part) {
  // da_part != null: also accumulate [da_s; da_d] = Σ_u [dp_u; dq_u] h̄_u per warp (fixed
  // node assignment) into da_part[block][2][D] for a fixed-order reduction.  These sums
  // cancel heavily (dp, dq and h̄ are signed), so they accumulate in float64.
  constexpr int V = D / 32;
  const int lane = threadIdx.x & 31;
  const int warps = (gridDim.x * NT) / 32;
  double das[V], dad[V];
  float a_sv[V], a_dv[V];
#pragma unroll
  for (int c = 0; c < V; ++c) {
    das[c] = dad[c] = 0.0;
    a_sv[c] = __ldg(a_s + lane * V + c);
    a_dv[c] = __ldg(a_d + lane * V + c);
  }
  for (int u = (blockIdx.x * NT + threadIdx.x) / 32; u < N; u += warps) {
    float acc[V];
#pragma unroll
    for (int c = 0; c < V; ++c) acc[c] = 0.f;
    float dp = 0.f, dq = 0.f;
    const int ob = __ldg(out_ptr + u), oe = __ldg(out_ptr + u + 1);
    // out-edge rows four at a time, all loads in flight (indices clamped into the segment;
    // surplus rows are never added), summed in ascending out-CSR order
    constexpr int G = 4;
    for (int j = ob; j < oe; j += G) {
      int kk[G];
      RawRow<V, false> rr[G];
      float da[G];
#pragma unroll
      for (int u2 = 0; u2 < G; ++u2) kk[u2] = __ldg(out_pos + min(j + u2, oe - 1));
#pragma unroll
      for (int u2 = 0; u2 < G; ++u2) {
        rr[u2].load(MG, long(kk[u2]), D, lane);
        da[u2] = __ldg(dalpha + kk[u2]);
      }
#pragma unroll
      for (int u2 = 0; u2 < G; ++u2) {
        if (j + u2 < oe) {
          float x[V];
          rr[u2].get(x);
#pragma unroll
          for (int c = 0; c < V; ++c) acc[c] += x[c];
          dp += da[u2];
        }
      }
    }
    for (int k = __ldg(in_ptr + u); k < __ldg(in_ptr + u + 1); ++k) dq += __ldg(dalpha + k);
    float hb[V], o[V];
    {
      RawRow<V, BF> hr;
      hr.load(hbar, long(u), D, lane);
      hr.get(hb);
    }
#pragma unroll
    for (int c = 0; c < V; ++c) {
      const int ch = lane * V + c;
      const float v = acc[c] + dp * a_sv[c] + dq * a_dv[c];
      o[c] = v * lrelu_grad_from_out(hb[c], slope);
      das[c] = fma(double(dp), double(hb[c]), das[c]);
      dad[c] = fma(double(dq), double(hb[c]), dad[c]);
      (void)ch;
    }
    store_row<V>(dP + long(u) * D + lane * V, o);
    if (lane == 0) {
      dpq[2 * long(u)] = dp;
      dpq[2 * long(u) + 1] = dq;
    }
  }
  if (da_part) {   // per-block partial: warps combined in fixed warp order through smem
    __shared__ double red[NT / 32][2 * D];
    const int wl = threadIdx.x / 32;
#pragma unroll
    for (int c = 0; c < V; ++c) {
      red[wl][lane * V + c] = das[c];
      red[wl][D + lane * V + c] = dad[c];
    }
    __syncthreads();
    for (int o = threadIdx.x; o < 2 * D; o += NT) {
      double acc2 = 0.0;
      for (int w2 = 0; w2 < NT / 32; ++w2) acc2 += red[w2][o];
      da_part[long(blockIdx.x) * 2 * D + o] = float(acc2);
    }
  }
}

// node_bwd with deeper memory-level parallelism (same sums, same per-node order): a warp
// takes chunks of 8 consecutive nodes; their out_ptr / in_ptr words, h̄ rows and in-edge dα
// sums are requested at once, then the chunk's out-edges (contiguous in out-CSR order) are
// walked G at a time with all G MG rows in flight, and each node is flushed as its out-edge
// segment ends (ascending out-CSR order, as node_bwd_kernel).
// FROMG: MG_k = dA[t_k] ⊙ g_k is formed here from the saved gates (g: BF16 rows when BF) and
// the layer's dA instead of being written by the gate backward and read back (the same FP32
// product, so the same bits).
// CPA (FROMG only): each out-edge's dA and g rows land in a per-warp shared-memory ring of
// NB_RING slots by cp.async (up to NB_RING edges in flight per warp, no registers held for
// them); the same rows are summed in the same order as the register path (bitwise equal).
// Ring depth x CTAs per SM measured on CFG3 (8x2: 3.62 ms, 6x3: 3.06, 5x3: 3.06, 7x3: 3.57,
// 4x4 with spills: 3.76, 12x2: 4.06; the register path 3.99).
#ifndef OCCU_NB_RING
#define OCCU_NB_RING 6
#endif
constexpr int NB_RING = OCCU_NB_RING;
template <int D, bool BF> constexpr int nb_slot_bytes() { return D * 4 + D * (BF ? 2 : 4); }

#ifndef OCCU_NB_CPA_MINB
#define OCCU_NB_CPA_MINB 3
#endif
template <int D, bool BF, bool FROMG, bool CPA = false>
__global__ void __launch_bounds__(NT, CPA ? OCCU_NB_CPA_MINB : (FROMG ? 2 : 3)) node_bwd_v2_kernel(
    const float *__restrict__ MG, const float *__restrict__ dalpha,
    const void *__restrict__ hbar, const float *__restrict__ a_s, const float *__restrict__ a_d,
    const int32_t *__restrict__ out_ptr, const int32_t *__restrict__ out_pos,
    const int32_t *__restrict__ in_ptr, int N, float slope, float *__restrict__ dP,
    float *__restrict__ dpq, float *__restrict__ da_part, const void *__restrict__ gsv,
    const float *__restrict__ dA, const int32_t *__restrict__ in_dst, int *__restrict__ dp_rexp) {
  // dp_rexp: the fp16x2 scale exponent of each dP row, for the dh_prev row-GEMM's converters
  constexpr int V = D / 32;
  constexpr int NPW = 8, G = 4;
  const int lane = threadIdx.x & 31;
  const long nw = (long(gridDim.x) * NT) / 32;
  double das[V], dad[V];
  float a_sv[V], a_dv[V];
#pragma unroll
  for (int c = 0; c < V; ++c) {
    das[c] = dad[c] = 0.0;
    a_sv[c] = __ldg(a_s + lane * V + c);
    a_dv[c] = __ldg(a_d + lane * V + c);
  }
  for (long t0 = (blockIdx.x * long(NT) + threadIdx.x) / 32 * NPW; t0 < N; t0 += nw * NPW) {
    const int nn = int(min(long(NPW), N - t0));
    const int op_l = lane <= nn ? __ldg(out_ptr + t0 + lane) : 0;
    const int ip_l = lane <= nn ? __ldg(in_ptr + t0 + lane) : 0;
    // h̄ row of the node being accumulated (the next one is requested at each flush) and dq
    // of node `lane` (lane < nn)
    RawRow<V, BF> hb;
    hb.load(hbar, t0, D, lane);
    float dq_l = 0.f;
    {
      const int ie = __shfl_down_sync(0xffffffffu, ip_l, 1);
      if (lane < nn)
        for (int k = ip_l; k < ie; ++k) dq_l += __ldg(dalpha + k);
    }
    const int e_beg = __shfl_sync(0xffffffffu, op_l, 0);
    const int e_end = __shfl_sync(0xffffffffu, op_l, nn);
    int node = 0;
    int seg_end = __shfl_sync(0xffffffffu, op_l, 1);
    float acc[V], dp = 0.f;
#pragma unroll
    for (int c = 0; c < V; ++c) acc[c] = 0.f;
    auto flush = [&](int nd) {
      float hv[V], o[V];
      hb.get(hv);
      if (nd + 1 < nn) hb.load(hbar, t0 + nd + 1, D, lane);
      const float dq = __shfl_sync(0xffffffffu, dq_l, nd);
#pragma unroll
      for (int c = 0; c < V; ++c) {
        const float v = acc[c] + dp * a_sv[c] + dq * a_dv[c];
        o[c] = v * lrelu_grad_from_out(hv[c], slope);
        das[c] = fma(double(dp), double(hv[c]), das[c]);
        dad[c] = fma(double(dq), double(hv[c]), dad[c]);
        acc[c] = 0.f;
      }
      store_row<V>(dP + (t0 + nd) * D + lane * V, o);
      if (lane == 0) {
        dpq[2 * (t0 + nd)] = dp;
        dpq[2 * (t0 + nd) + 1] = dq;
      }
      if (dp_rexp) {          // row max |dP|: one warp integer max-reduce of the |x| bit patterns
        float mx = 0.f;
#pragma unroll
        for (int c = 0; c < V; ++c) mx = fmaxf(mx, fabsf(o[c]));
        mx = __uint_as_float(__reduce_max_sync(0xffffffffu, __float_as_uint(mx)));
        if (lane == 0) dp_rexp[t0 + nd] = occu_row_scale_exp(mx);
      }
      dp = 0.f;
    };
    for (int base = e_beg; base < e_end; base += 32) {
      const int cnt = min(32, e_end - base);
      const int pos_l = lane < cnt ? __ldg(out_pos + base + lane) : 0;
      const float da_l = lane < cnt ? __ldg(dalpha + pos_l) : 0.f;
      const int dst_l = (FROMG && lane < cnt) ? __ldg(in_dst + pos_l) : 0;
      if constexpr (CPA && FROMG) {
        extern __shared__ __align__(16) uint8_t nb_dyn[];
        constexpr int SLOT = nb_slot_bytes<D, BF>(), GB = BF ? 2 : 4;
        uint8_t *ring = nb_dyn + (threadIdx.x / 32) * (NB_RING * SLOT);
        auto issue = [&](int jj) {                   // edge jj of the batch -> slot jj % NB_RING
          if (jj < cnt) {
            const long ps = __shfl_sync(0xffffffffu, pos_l, jj), ds = __shfl_sync(0xffffffffu, dst_l, jj);
            uint8_t *sp = ring + (jj % NB_RING) * SLOT;
            cpa_ca<V * 4>(sp + lane * V * 4, dA + ds * D + lane * V);
            cpa_ca<V * GB>(sp + D * 4 + lane * V * GB,
                           reinterpret_cast<const uint8_t *>(gsv) + (ps * D + lane * V) * GB);
          }
          cpa_commit_nb();                             // one group per edge slot, empty past cnt
        };
#pragma unroll
        for (int q = 0; q < NB_RING; ++q) issue(q);
        for (int j = 0; j < cnt; ++j) {
          cpa_wait_nb<NB_RING - 1>();                  // edge j's group has landed (lane-private rows)
          const float dau = __shfl_sync(0xffffffffu, da_l, j);
          const int k = base + j;
          while (k >= seg_end) {
            flush(node);
            ++node;
            seg_end = __shfl_sync(0xffffffffu, op_l, node + 1);
          }
          const uint8_t *sp = ring + (j % NB_RING) * SLOT;
          float x[V], gv[V];
#pragma unroll
          for (int c = 0; c < V; ++c) x[c] = reinterpret_cast<const float *>(sp)[lane * V + c];
          if constexpr (BF) {
#pragma unroll
            for (int c = 0; c < V; ++c)
              gv[c] = __uint_as_float(uint32_t(reinterpret_cast<const uint16_t *>(sp + D * 4)[lane * V + c]) << 16);
          } else {
#pragma unroll
            for (int c = 0; c < V; ++c) gv[c] = reinterpret_cast<const float *>(sp + D * 4)[lane * V + c];
          }
#pragma unroll
          for (int c = 0; c < V; ++c) acc[c] += x[c] * gv[c];     // dm ⊙ g, as the gate backward
          dp += dau;
          issue(j + NB_RING);
        }
        cpa_wait_nb<0>();
        continue;
      }
      for (int j = 0; j < cnt; j += G) {
        RawRow<V, false> rr[G];
        RawRow<V, BF> gg[FROMG ? G : 1];
#pragma unroll
        for (int u = 0; u < G; ++u) {
          const int kk = min(j + u, cnt - 1);
          if constexpr (FROMG) {
            gg[u].load(gsv, long(__shfl_sync(0xffffffffu, pos_l, kk)), D, lane);
            rr[u].load(dA, long(__shfl_sync(0xffffffffu, dst_l, kk)), D, lane);
          } else {
            rr[u].load(MG, long(__shfl_sync(0xffffffffu, pos_l, kk)), D, lane);
          }
        }
#pragma unroll
        for (int u = 0; u < G; ++u) {
          const float dau = __shfl_sync(0xffffffffu, da_l, min(j + u, cnt - 1));
          if (j + u < cnt) {
            const int k = base + j + u;
            while (k >= seg_end) {
              flush(node);
              ++node;
              seg_end = __shfl_sync(0xffffffffu, op_l, node + 1);
            }
            float x[V];
            rr[u].get(x);
            if constexpr (FROMG) {
              float gv[V];
              gg[u].get(gv);
#pragma unroll
              for (int c = 0; c < V; ++c) x[c] = x[c] * gv[c];     // dm ⊙ g, as the gate backward
            }
#pragma unroll
            for (int c = 0; c < V; ++c) acc[c] += x[c];
            dp += dau;
          }
        }
      }
    }
    for (; node < nn; ++node) flush(node);
  }
  if (da_part) {   // per-block partial: warps combined in fixed warp order through smem
    __shared__ double red[NT / 32][2 * D];
    const int wl = threadIdx.x / 32;
#pragma unroll
    for (int c = 0; c < V; ++c) {
      red[wl][lane * V + c] = das[c];
      red[wl][D + lane * V + c] = dad[c];
    }
    __syncthreads();
    for (int o = threadIdx.x; o < 2 * D; o += NT) {
      double acc2 = 0.0;
      for (int w2 = 0; w2 < NT / 32; ++w2) acc2 += red[w2][o];
      da_part[long(blockIdx.x) * 2 * D + o] = float(acc2);
    }
  }
}

// Deterministic split-K weight gradient: partial[s][a][b] = Σ_{r in split s} X[r][a] Y[r][b]
// (X: [R][A], Y: [R][Bn]; 128x128 output tile per CTA, 8x8 per thread).
constexpr int WG_R = 32;
__global__ void __launch_bounds__(NT) wgrad_partial_kernel(const float *__restrict__ X, int A,
                                                           const float *__restrict__ Y, int Bn,
                                                           long R, int splits,
                                                           float *__restrict__ partial) {
  __shared__ __align__(16) float Xs[WG_R][128];
  __shared__ __align__(16) float Ys[WG_R][128];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int s = blockIdx.x;
  const int a0 = blockIdx.y * 128, b0 = blockIdx.z * 128;
  const long per = (R + splits - 1) / splits;
  const long r0 = s * per, r1 = min(R, r0 + per);
  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  for (long rb = r0; rb < r1; rb += WG_R) {
    __syncthreads();
    for (int idx = threadIdx.x; idx < WG_R * 128; idx += NT) {
      const int rr = idx / 128, cc = idx % 128;
      const long row = rb + rr;
      const bool ok = row < r1;
      Xs[rr][cc] = (ok && a0 + cc < A) ? X[row * A + a0 + cc] : 0.f;
      Ys[rr][cc] = (ok && b0 + cc < Bn) ? Y[row * Bn + b0 + cc] : 0.f;
    }
    __syncthreads();
#pragma unroll 4
    for (int rr = 0; rr < WG_R; ++rr) {
      const float4 x0 = *reinterpret_cast<const float4 *>(&Xs[rr][ty * 4]);
      const float4 x1 = *reinterpret_cast<const float4 *>(&Xs[rr][64 + ty * 4]);
      const float4 y0 = *reinterpret_cast<const float4 *>(&Ys[rr][tx * 4]);
      const float4 y1 = *reinterpret_cast<const float4 *>(&Ys[rr][64 + tx * 4]);
      const float xv[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
      const float yv[8] = {y0.x, y0.y, y0.z, y0.w, y1.x, y1.y, y1.z, y1.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(xv[i], yv[j], acc[i][j]);
    }
  }
  float *out = partial + long(s) * A * Bn;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int a = a0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
    if (a >= A) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int b = b0 + (j < 4 ? tx * 4 + j : 64 + tx * 4 + j - 4);
      if (b < Bn) out[long(a) * Bn + b] = acc[i][j];
    }
  }
}

// Skinny weight gradients (A*Bn <= 512, e.g. dW_e of layer 1 with F_e = 4, [da_s; da_d]):
// thread o owns outputs o and o+256; rows staged through smem in chunks of 32.
__global__ void __launch_bounds__(NT) wgrad_skinny_kernel(const float *__restrict__ X, int A,
                                                          const float *__restrict__ Y, int Bn,
                                                          long R, int splits,
                                                          float *__restrict__ partial) {
  __shared__ float Xs[WG_R][129];
  __shared__ float Ys[WG_R][129];
  const int n = A * Bn;
  const long per = (R + splits - 1) / splits;
  const long r0 = blockIdx.x * per, r1 = min(R, r0 + per);
  float acc0 = 0.f, acc1 = 0.f;
  const int o0 = threadIdx.x, o1 = threadIdx.x + NT;
  const int a0 = o0 / Bn, b0 = o0 % Bn, a1 = o1 / Bn, b1 = o1 % Bn;
  for (long rb = r0; rb < r1; rb += WG_R) {
    __syncthreads();
    for (int idx = threadIdx.x; idx < WG_R * A; idx += NT) {
      const int rr = idx / A, cc = idx % A;
      Xs[rr][cc] = rb + rr < r1 ? X[(rb + rr) * A + cc] : 0.f;
    }
    for (int idx = threadIdx.x; idx < WG_R * Bn; idx += NT) {
      const int rr = idx / Bn, cc = idx % Bn;
      Ys[rr][cc] = rb + rr < r1 ? Y[(rb + rr) * Bn + cc] : 0.f;
    }
    __syncthreads();
    if (o0 < n)
      for (int rr = 0; rr < WG_R; ++rr) acc0 = fmaf(Xs[rr][a0], Ys[rr][b0], acc0);
    if (o1 < n)
      for (int rr = 0; rr < WG_R; ++rr) acc1 = fmaf(Xs[rr][a1], Ys[rr][b1], acc1);
  }
  float *out = partial + long(blockIdx.x) * n;
  if (o0 < n) out[o0] = acc0;
  if (o1 < n) out[o1] = acc1;
}

// out[o] = Σ_k partial[k][o] with the split range cut into LANES interleaved
// sub-sums (lane l takes k ≡ l mod LANES) combined in lane order: fixed order,
// LANES-way parallel per output.
template <int LANES>
__global__ void __launch_bounds__(256) split_reduce_kernel(const float *__restrict__ partial,
                                                           int splits, long n,
                                                           float *__restrict__ out) {
  constexpr int OPB = 256 / LANES;            // outputs per block
  __shared__ float red[LANES][OPB];
  const int ol = threadIdx.x % OPB, l = threadIdx.x / OPB;
  const long o = long(blockIdx.x) * OPB + ol;
  float acc = 0.f;
  if (o < n)
    for (int k = l; k < splits; k += LANES) acc += partial[long(k) * n + o];
  red[l][ol] = acc;
  __syncthreads();
  if (l == 0 && o < n) {
    float t = 0.f;
    for (int j = 0; j < LANES; ++j) t += red[j][ol];
    out[o] = t;
  }
}

// Several split-K reductions in one launch (the weight gradients of one layer and the
// [da_s; da_d] partials): job j owns blocks [blk[j], blk[j+1]); within a job the order is
// split_reduce_kernel's (fixed, deterministic).
struct ReduceJob { const float *part; float *out; long n; int splits; int lanes = 8; };
struct ReduceJobs { ReduceJob j[4]; int blk[5]; int count; };
// job.lanes threads per output (8 for 128x128 weight gradients, 64 for the few outputs of
// [da_s; da_d] with thousands of partials), 256 / lanes outputs per block.
__global__ void __launch_bounds__(256) multi_reduce_kernel(const ReduceJobs jobs) {
  __shared__ double red[256];   // partial sums of signed gradients cancel: float64
  int q = 0;
  while (q + 1 < jobs.count && int(blockIdx.x) >= jobs.blk[q + 1]) ++q;
  const ReduceJob jb = jobs.j[q];
  const int lanes = jb.lanes, opb = 256 / lanes;
  const int ol = threadIdx.x % opb, l = threadIdx.x / opb;
  const long o = long(int(blockIdx.x) - jobs.blk[q]) * opb + ol;
  double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;     // four independent chains in flight
  if (o < jb.n) {
    int k = l;
    for (; k + 3 * lanes < jb.splits; k += 4 * lanes) {
      a0 += __ldg(jb.part + long(k) * jb.n + o);
      a1 += __ldg(jb.part + long(k + lanes) * jb.n + o);
      a2 += __ldg(jb.part + long(k + 2 * lanes) * jb.n + o);
      a3 += __ldg(jb.part + long(k + 3 * lanes) * jb.n + o);
    }
    for (; k < jb.splits; k += lanes) a0 += __ldg(jb.part + long(k) * jb.n + o);
  }
  red[l * opb + ol] = (a0 + a1) + (a2 + a3);
  __syncthreads();
  if (l == 0 && o < jb.n) {
    double t = 0.0;
    for (int x = 0; x < lanes; ++x) t += red[x * opb + ol];
    jb.out[o] = float(t);
  }
}

__global__ void wgrad_reduce_kernel(const float *__restrict__ partial, int splits, long n,
                                    float *__restrict__ out) {
  for (long i = blockIdx.x * long(blockDim.x) + threadIdx.x; i < n; i += long(gridDim.x) * blockDim.x) {
    double s = 0.0;
    for (int k = 0; k < splits; ++k) s += partial[long(k) * n + i];
    out[i] = float(s);
  }
}

// a12: Adam, PyTorch semantics (R16).
__global__ void adam_kernel(float *__restrict__ w, const float *__restrict__ g, float *__restrict__ m,
                            float *__restrict__ v, long n, float lr, float wd, float b1, float b2,
                            float bc1, float bc2, float eps) {
  for (long i = blockIdx.x * long(blockDim.x) + threadIdx.x; i < n; i += long(gridDim.x) * blockDim.x) {
    const float gr = g[i] + wd * w[i];
    const float mi = b1 * m[i] + (1.f - b1) * gr;
    const float vi = b2 * v[i] + (1.f - b2) * gr * gr;
    m[i] = mi;
    v[i] = vi;
    const float mhat = mi / bc1;
    const float vhat = vi / bc2;
    w[i] = w[i] - lr * mhat / (sqrtf(vhat) + eps);
  }
}

inline int grid_for(long work, int per_block, int cap) {
  long g = (work + per_block - 1) / per_block;
  if (g < 1) g = 1;
  if (g > cap) g = cap;
  return int(g);
}

template <class K> cudaError_t set_smem(K kern, size_t bytes) {
  return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes));
}

}  // namespace

// ---------------------------------------------------------------------------
// Launchers
// ---------------------------------------------------------------------------
#define LAUNCH_CHECK()                                  \
  do {                                                  \
    cudaError_t e_ = cudaGetLastError();                \
    if (e_ != cudaSuccess) return -int(e_);             \
  } while (0)

template <int D>
static int forward_layer_impl(const occu_ctx *ctx, const DevCsr &csr, const FwdLayerArgs &a,
                              cudaStream_t st) {
  const int sms = ctx->num_sms;
  int n = 0;
  if (csr.N > 0) {
    const size_t sm1 = (size_t(a.K) * D + BM * (a.K + 4)) * 4;
    set_smem(node_gemm_kernel<D, 0>, sm1);
    const int tiles = (csr.N + BM - 1) / BM;
    OCCU_PROF_BEGIN(ctx, "node_gemm", st);
    node_gemm_kernel<D, 0><<<grid_for(tiles, 1, 2 * sms), NT, sm1, st>>>(
        a.h_in, a.K, a.W_u, a.a_s, a.a_d, csr.N, ctx->cfg.slope, a.hbar, a.p, a.q);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    ++n;
  }
  if (csr.E > 0) {
    const size_t sm2 = (size_t(a.Ke) * D + D * D + BM * (a.Ke + 4) + BM * (D + 4) + BM) * 4;
    set_smem(edge_fwd_kernel<D>, sm2);
    const int tiles = (csr.E + BM - 1) / BM;
    OCCU_PROF_BEGIN(ctx, "edge_fwd", st);
    edge_fwd_kernel<D><<<grid_for(tiles, 1, sms), NT, sm2, st>>>(
        a.e_in, a.Ke, a.W_e, a.W_m, a.p, a.q, csr.in_src, csr.in_dst, csr.E, a.e_out, a.g);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    ++n;
  }
  if (csr.N > 0) {
    OCCU_PROF_BEGIN(ctx, "gather_segsum", st);
    gather_segsum_kernel<D, false><<<grid_for(long(csr.N) * 4, NT, 16 * sms), NT, 0, st>>>(
        a.g, a.hbar, csr.in_ptr, csr.in_src, csr.N, ctx->cfg.aggr == OCCU_AGGR_MEAN,
        ctx->cfg.slope, a.h_out, nullptr, nullptr);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    ++n;
  }
  return n;
}

// Hub pre-pass of the aggregation (hub_partial_kernel + hub_merge_kernel) when the batch has
// destinations of in-degree > HUB_DEG (or its maximum is unknown); *hub = the unit sums.
template <int D, bool BF>
static int launch_hub_sums(const occu_ctx *ctx, const DevCsr &csr, const void *g, const void *hbar,
                           const float **hub, cudaStream_t st) {
  *hub = nullptr;
  if (csr.E <= 0 || (csr.max_deg >= 0 && csr.max_deg <= HUB_DEG)) return 0;
  const long units = (long(csr.E) + HUB_UB - 1) / HUB_UB;
  if (const_cast<occu_ctx *>(ctx)->ws.hub.ensure(size_t(units) * 2 * D * 4) != cudaSuccess)
    return -int(cudaErrorMemoryAllocation);
  float *part = ctx->ws.hub.as<float>();
  const int grid = grid_for(units * 32, NT, 8 * ctx->num_sms);
  OCCU_PROF_BEGIN(ctx, "gather_hubs", st);
  hub_partial_kernel<D, BF><<<grid, NT, 0, st>>>(g, hbar, csr.in_ptr, csr.in_src, csr.in_dst, csr.E, part);
  hub_merge_kernel<D><<<grid, NT, 0, st>>>(csr.in_ptr, csr.in_dst, csr.E, part);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  *hub = part;
  return 2;
}

template <int D>
static int gather_impl(const occu_ctx *ctx, const DevCsr &csr, const float *g, const float *hbar,
                       float *h_out, float *rpart, cudaStream_t st, uint32_t *hbits) {
  if (csr.N <= 0) return 0;
  static const int variant = [] {
    const char *e = getenv("OCCU_GATHER_V");
    return e ? atoi(e) : 1;
  }();
  static const int occ = [] {
    const char *e = getenv("OCCU_GATHER_BPS");
    return e ? atoi(e) : 8;
  }();
  const int mean = ctx->cfg.aggr == OCCU_AGGR_MEAN;
  const float *hub = nullptr;
  int r0 = launch_hub_sums<D, false>(ctx, csr, g, hbar, &hub, st);
  if (r0 < 0) return r0;
  OCCU_PROF_BEGIN(ctx, "gather_segsum", st);
#define OCCU_GATHER_ARGS g, hbar, csr.in_ptr, csr.in_src, csr.N, mean, ctx->cfg.slope, h_out, csr.node_graph, rpart, hub, csr.in_dst, hbits
  if (hbits && variant != 1) return -int(cudaErrorInvalidValue);    // sign bits: default kernel only
  if (hbits) {                // training forward: the sign-bit variants
    const int grid = grid_for(long(csr.N) * 4, NT, occ * ctx->num_sms);
    constexpr int GG = D == 256 ? 2 : 4;
    if (rpart) launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, GG, true, false, false, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
    else launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, GG, false, false, false, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
  } else if constexpr (D == 256) {
    // d = 256: two (g, h̄) row pairs in flight per lane (16 floats each); 1 KB rows
    const int grid = grid_for(long(csr.N) * 4, NT, occ * ctx->num_sms);
    if (rpart) launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 2, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
    else launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 2, false>, grid, NT, 0, st, OCCU_GATHER_ARGS);
  } else if (variant == 0) {
    const int grid = grid_for(long(csr.N) * 4, NT, 16 * ctx->num_sms);
#define OCCU_GATHER_ARGS0 g, hbar, csr.in_ptr, csr.in_src, csr.N, mean, ctx->cfg.slope, h_out, csr.node_graph, rpart
    if (rpart) gather_segsum_kernel<D, true><<<grid, NT, 0, st>>>(OCCU_GATHER_ARGS0);
    else gather_segsum_kernel<D, false><<<grid, NT, 0, st>>>(OCCU_GATHER_ARGS0);
#undef OCCU_GATHER_ARGS0
  } else {
    const int grid = grid_for(long(csr.N) * 4, NT, occ * ctx->num_sms);
    if (variant == 1) {
      if (rpart) launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 4, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
      else launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 4, false>, grid, NT, 0, st, OCCU_GATHER_ARGS);
    } else if (variant == 3) {
      if (rpart) launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 4, true, false, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
      else launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 4, false, false, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
    } else if (variant == 4) {
      if (rpart) launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 2, true, false, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
      else launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 2, false, false, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
    } else {
      if (rpart) launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 8, true>, grid, NT, 0, st, OCCU_GATHER_ARGS);
      else launch_pdl(ctx->pdl & 2, gather_segsum_v2_kernel<D, 8, false>, grid, NT, 0, st, OCCU_GATHER_ARGS);
    }
  }
#undef OCCU_GATHER_ARGS
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1 + r0;
}

template <int D>
static int gather_bf16_impl(const occu_ctx *ctx, const DevCsr &csr, const void *g, const void *hbar,
                            void *h_out, float *rpart, cudaStream_t st, uint32_t *hbits) {
  if (csr.N <= 0) return 0;
  const int mean = ctx->cfg.aggr == OCCU_AGGR_MEAN;
  static const int gsel = [] {
    const char *e = getenv("OCCU_GATHER_G");
    return e ? atoi(e) : 4;
  }();
  static const int bps = [] {
    const char *e = getenv("OCCU_GATHER_BPS");
    return e ? atoi(e) : 8;
  }();
  const int grid = grid_for(long(csr.N) * 4, NT, bps * ctx->num_sms);
  const float *hub = nullptr;
  int r0 = launch_hub_sums<D, true>(ctx, csr, g, hbar, &hub, st);
  if (r0 < 0) return r0;
  OCCU_PROF_BEGIN(ctx, "gather_segsum", st);
#define OCCU_GB_ARGS g, hbar, csr.in_ptr, csr.in_src, csr.N, mean, ctx->cfg.slope, h_out, csr.node_graph, rpart, hub, csr.in_dst, hbits
  if (hbits) {                // training forward: the sign-bit variants
    constexpr int GG = D == 256 ? 2 : 4;
    if (rpart) launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, GG, true, true, false, true>, grid, NT, 0, st, OCCU_GB_ARGS);
    else launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, GG, false, true, false, true>, grid, NT, 0, st, OCCU_GB_ARGS);
  } else if constexpr (D == 256) {
    if (rpart) launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 2, true, true>, grid, NT, 0, st, OCCU_GB_ARGS);
    else launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 2, false, true>, grid, NT, 0, st, OCCU_GB_ARGS);
  } else if (gsel == 4) {
    if (rpart) launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 4, true, true>, grid, NT, 0, st, OCCU_GB_ARGS);
    else launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 4, false, true>, grid, NT, 0, st, OCCU_GB_ARGS);
  } else if (gsel == 2) {
    if (rpart) launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 2, true, true, true>, grid, NT, 0, st, OCCU_GB_ARGS);
    else launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 2, false, true, true>, grid, NT, 0, st, OCCU_GB_ARGS);
  } else {
    if (rpart) launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 4, true, true, true>, grid, NT, 0, st, OCCU_GB_ARGS);
    else launch_pdl(ctx->pdl & 64, gather_segsum_v2_kernel<D, 4, false, true, true>, grid, NT, 0, st, OCCU_GB_ARGS);
  }
#undef OCCU_GB_ARGS
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1 + r0;
}

template <int D, bool BF>
static int segsoftmax_impl(const occu_ctx *ctx, const DevCsr &csr, void *v, const void *hbar,
                           void *h_out, float *rpart, bool write_w, cudaStream_t st) {
  if (csr.N <= 0) return 0;
  const int mean = ctx->cfg.aggr == OCCU_AGGR_MEAN;
  const int grid = grid_for(long(csr.N) * 4, NT, 8 * ctx->num_sms);
  OCCU_PROF_BEGIN(ctx, "gather_segsoftmax", st);
#define OCCU_GS_ARGS v, hbar, csr.in_ptr, csr.in_src, csr.N, mean, ctx->cfg.slope, h_out, csr.node_graph, rpart
  if (write_w) {
    if (rpart) launch_pdl(ctx->pdl & 2, gather_segsoftmax_kernel<D, 4, true, true, BF>, grid, NT, 0, st, OCCU_GS_ARGS);
    else launch_pdl(ctx->pdl & 2, gather_segsoftmax_kernel<D, 4, false, true, BF>, grid, NT, 0, st, OCCU_GS_ARGS);
  } else {
    if (rpart) launch_pdl(ctx->pdl & 2, gather_segsoftmax_kernel<D, 4, true, false, BF>, grid, NT, 0, st, OCCU_GS_ARGS);
    else launch_pdl(ctx->pdl & 2, gather_segsoftmax_kernel<D, 4, false, false, BF>, grid, NT, 0, st, OCCU_GS_ARGS);
  }
#undef OCCU_GS_ARGS
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1;
}

int launch_gather_segsoftmax(const occu_ctx *ctx, const DevCsr &csr, float *v, const float *hbar,
                             float *h_out, float *rpart, bool write_w, cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return segsoftmax_impl<64, false>(ctx, csr, v, hbar, h_out, rpart, write_w, st);
    case 128: return segsoftmax_impl<128, false>(ctx, csr, v, hbar, h_out, rpart, write_w, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

// OCCU_BF16 reading B: BF16 logits / weights v, h̄ and h
int launch_gather_segsoftmax_bf16(const occu_ctx *ctx, const DevCsr &csr, void *v, const void *hbar,
                                  void *h_out, float *rpart, bool write_w, cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return segsoftmax_impl<64, true>(ctx, csr, v, hbar, h_out, rpart, write_w, st);
    case 128: return segsoftmax_impl<128, true>(ctx, csr, v, hbar, h_out, rpart, write_w, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

int launch_gather_segsum_bf16(const occu_ctx *ctx, const DevCsr &csr, const void *g,
                              const void *hbar, void *h_out, float *rpart, cudaStream_t st,
                              uint32_t *h_bits) {
  switch (ctx->cfg.d) {
    case 64: return gather_bf16_impl<64>(ctx, csr, g, hbar, h_out, rpart, st, h_bits);
    case 128: return gather_bf16_impl<128>(ctx, csr, g, hbar, h_out, rpart, st, h_bits);
    case 256: return gather_bf16_impl<256>(ctx, csr, g, hbar, h_out, rpart, st, h_bits);
    default: return -int(cudaErrorInvalidValue);
  }
}

int launch_gather_segsum(const occu_ctx *ctx, const DevCsr &csr, const float *g,
                         const float *hbar, float *h_out, float *rpart, cudaStream_t st,
                         uint32_t *h_bits) {
  switch (ctx->cfg.d) {
    case 64: return gather_impl<64>(ctx, csr, g, hbar, h_out, rpart, st, h_bits);
    case 128: return gather_impl<128>(ctx, csr, g, hbar, h_out, rpart, st, h_bits);
    case 256: return gather_impl<256>(ctx, csr, g, hbar, h_out, rpart, st, h_bits);
    default: return -int(cudaErrorInvalidValue);
  }
}

int launch_forward_layer(const occu_ctx *ctx, const DevCsr &csr, const FwdLayerArgs &a,
                         cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return forward_layer_impl<64>(ctx, csr, a, st);
    case 128: return forward_layer_impl<128>(ctx, csr, a, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

int launch_permute_rows(const occu_ctx *ctx, const float *src, const int32_t *idx, int rows,
                        int width, float *dst, cudaStream_t st) {
  if (rows <= 0) return 0;
  OCCU_PROF_BEGIN(ctx, "permute_e0", st);
  permute_rows_kernel<<<grid_for(long(rows) * width, 256, 4096), 256, 0, st>>>(src, idx, rows,
                                                                                width, dst);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1;
}

int launch_readout_head(const occu_ctx *ctx, const DevCsr &csr, const float *h, bool chunked,
                        const float *params, float *r, float *c, float *yhat, cudaStream_t st) {
  const occu_config &cf = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  const size_t smem = (RO_WARPS * cf.d + cf.d + cf.d_h) * 4;
  OCCU_PROF_BEGIN(ctx, "readout_head", st);
#define OCCU_RO_ARGS h, csr.node_off, cf.d_h, params + L.W_1, params + L.b_1, params + L.w_2, \
    params + L.b_2, cf.slope, r, c, yhat, chunked ? 8 : 0
  if (cf.d == 64) launch_pdl(ctx->pdl & 8, readout_head_kernel<64>, csr.B, RO_WARPS * 32, smem, st, OCCU_RO_ARGS);
  else if (cf.d == 128) launch_pdl(ctx->pdl & 8, readout_head_kernel<128>, csr.B, RO_WARPS * 32, smem, st, OCCU_RO_ARGS);
  else launch_pdl(ctx->pdl & 8, readout_head_kernel<256>, csr.B, RO_WARPS * 32, smem, st, OCCU_RO_ARGS);
#undef OCCU_RO_ARGS
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1;
}

static int reduce_splits(const occu_ctx *ctx, const float *part, int splits, long n, float *out,
                         cudaStream_t st) {
  OCCU_PROF_BEGIN(ctx, "split_reduce", st);
  if (n >= 4096)
    split_reduce_kernel<8><<<int((n + 31) / 32), 256, 0, st>>>(part, splits, n, out);
  else
    split_reduce_kernel<64><<<int((n + 3) / 4), 256, 0, st>>>(part, splits, n, out);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1;
}

// Partial-sum slots of the deferred weight gradients: one per GEMM of a layer + the
// [da_s; da_d] partials, each up to 2·148 splits x 128 x 128 floats.
constexpr size_t WG_SLOT_FLOATS = size_t(2 * 160) * 128 * 128;

static int launch_multi_reduce(const occu_ctx *ctx, ReduceJobs &rj, cudaStream_t st) {
  if (rj.count == 0) return 0;
  rj.blk[0] = 0;
  for (int q = 0; q < rj.count; ++q) {
    rj.j[q].lanes = rj.j[q].n >= 4096 ? 8 : 64;
    const int opb = 256 / rj.j[q].lanes;
    rj.blk[q + 1] = rj.blk[q] + int((rj.j[q].n + opb - 1) / opb);
  }
  OCCU_PROF_BEGIN(ctx, "split_reduce", st);
  multi_reduce_kernel<<<rj.blk[rj.count], 256, 0, st>>>(rj);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  rj.count = 0;
  return 1;
}

static int wgrad_impl(occu_ctx *ctx, const float *X, int A, const void *Yv, int Bn, long R,
                      float *out, cudaStream_t st, bool ybf, ReduceJobs *defer, float *slot);

// ybf: Y holds BF16 rows (OCCU_BF16 training); only the tensor-core kernel reads those.
static int wgrad(occu_ctx *ctx, const float *X, int A, const void *Yv, int Bn, long R, float *out,
                 cudaStream_t st, bool ybf = false) {
  return wgrad_impl(ctx, X, A, Yv, Bn, R, out, st, ybf, nullptr, nullptr);
}

// Deferred: the partials go to `slot` and the reduction is appended to `rj` (one
// launch_multi_reduce per layer instead of one reduction launch per GEMM).
static int wgrad_deferred(occu_ctx *ctx, const float *X, int A, const void *Yv, int Bn, long R,
                          float *out, cudaStream_t st, bool ybf, ReduceJobs &rj, float *slot) {
  return wgrad_impl(ctx, X, A, Yv, Bn, R, out, st, ybf, &rj, slot);
}

static int wgrad_impl(occu_ctx *ctx, const float *X, int A, const void *Yv, int Bn, long R,
                      float *out, cudaStream_t st, bool ybf, ReduceJobs *defer, float *slot) {
  const float *Y = reinterpret_cast<const float *>(Yv);
  const long n = long(A) * Bn;
  const int ta = (A + 127) / 128, tb = (Bn + 127) / 128;
  int splits = int(std::max<long>(1, std::min<long>((2L * ctx->num_sms) / (ta * tb), (R + 255) / 256)));
  if (R == 0) {
    cudaMemsetAsync(out, 0, n * 4, st);
    return 0;
  }
  if (ybf && !wgrad_tc_supported(A, Bn)) return -int(cudaErrorInvalidValue);
  static const long tc_min = getenv("OCCU_WGRAD_TC_MIN") ? atol(getenv("OCCU_WGRAD_TC_MIN")) : 4096;
  auto get_part = [&](int sp) -> float * {
    if (defer) return slot;
    if (ctx->ws.partial.ensure(size_t(sp) * n * 4) != cudaSuccess) return nullptr;
    return ctx->ws.partial.as<float>();
  };
  auto finish = [&](float *part, int sp) -> int {
    if (defer) {
      defer->j[defer->count++] = ReduceJob{part, out, n, sp};
      return 0;
    }
    return reduce_splits(ctx, part, sp, n, out, st);
  };
  if (ctx->path != 1 && wgrad_tc_supported(A, Bn) && (R >= tc_min || ybf)) {
    const int sp = ctx->num_sms;
    float *part = get_part(sp);
    if (!part) return -int(cudaErrorMemoryAllocation);
    int r = launch_wgrad_tc(ctx, X, A, Yv, Bn, R, sp, part, st, ybf);
    if (r < 0) return r;
    return r + finish(part, sp);
  }
  if (n <= 2 * NT && A <= 128 && Bn <= 128) {
    const int sp = 2 * ctx->num_sms;
    float *part = get_part(sp);
    if (!part) return -int(cudaErrorMemoryAllocation);
    OCCU_PROF_BEGIN(ctx, "wgrad_skinny", st);
    wgrad_skinny_kernel<<<sp, NT, 0, st>>>(X, A, Y, Bn, R, sp, part);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    return 1 + finish(part, sp);
  }
  float *part = get_part(splits);
  if (!part) return -int(cudaErrorMemoryAllocation);
  OCCU_PROF_BEGIN(ctx, "wgrad_partial", st);
  wgrad_partial_kernel<<<dim3(splits, ta, tb), NT, 0, st>>>(X, A, Y, Bn, R, splits, part);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1 + finish(part, splits);
}

int launch_wgrad(occu_ctx *ctx, const float *X, int A, const void *Y, int Bn, long R, float *out,
                 cudaStream_t st, bool ybf) {
  return wgrad(ctx, X, A, Y, Bn, R, out, st, ybf);
}

int launch_head_backward(occu_ctx *ctx, const DevCsr &csr, const float *targets, int global_B,
                         cudaStream_t st) {
  static const bool use_bits = !getenv("OCCU_NO_HBITS");
  const occu_config &cf = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  Workspace &w = ctx->ws;
  float *P = ctx->params.as<float>();
  float *G = ctx->grads.as<float>();
  const float inv_gb = 1.f / float(global_B);
  OCCU_PROF_BEGIN(ctx, "head_bwd_graph", st);
  const int hin = L.head_in;          // d (mean readout) or k·d (decoder readout)
  head_bwd_graph_kernel<<<csr.B, 128, cf.d_h * 4, st>>>(
      w.yhat.as<float>(), targets, w.c.as<float>(), P + L.W_1, P + L.w_2, hin, cf.d_h, inv_gb,
      cf.slope, w.dy.as<float>(), w.dc.as<float>(), w.dr.as<float>());
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  const int jobs = cf.d_h * hin + 2 * cf.d_h + 2;
  OCCU_PROF_BEGIN(ctx, "head_bwd_reduce", st);
  head_bwd_reduce_kernel<<<grid_for(jobs, 256, 1024), 256, 0, st>>>(
      w.dy.as<float>(), w.dc.as<float>(), w.r.as<float>(), w.c.as<float>(), w.yhat.as<float>(),
      targets, csr.B, hin, cf.d_h, inv_gb, cf.slope, G + L.W_1, G + L.b_1, G + L.w_2, G + L.b_2,
      w.loss.as<float>());
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  if (cf.readout == OCCU_READOUT_SET_DECODER) return 2;   // dr feeds the decoder backward
  OCCU_PROF_BEGIN(ctx, "broadcast_dh", st);
  // TC backward consumes dA directly; with Graphormer layers dr/n_b is the gradient of the
  // stack's top states and the mask is applied below the stack (launch_mask_dA)
  const bool tcb = ctx->path != 1 && tc_supported(cf) && cf.graphormer == 0;
  const uint32_t *hl_bits = (tcb && use_bits && ctx->hbits_layers >= cf.L)
                                ? reinterpret_cast<const uint32_t *>(w.hbits[cf.L - 1].ptr) : nullptr;
  static const bool bdh4 = !getenv("OCCU_BDH_V1");        // A/B switch (bitwise-equal results)
  if (hl_bits && cf.d == 128 && bdh4) {
    broadcast_dh_bits128_kernel<<<grid_for((long(csr.N) + 3) / 4, 8, 8 * ctx->num_sms), 256, 0, st>>>(
        w.dr.as<float>(), csr.node_graph, csr.node_off, csr.N, csr.in_ptr, cf.aggr == OCCU_AGGR_MEAN,
        cf.slope, w.dh.as<float>(), hl_bits);
  } else
  broadcast_dh_kernel<<<grid_for(long(csr.N) * cf.d / 4, 256, 16 * ctx->num_sms), 256, 0, st>>>(
      w.dr.as<float>(), csr.node_graph, csr.node_off, csr.N, cf.d,
      tcb ? w.h[cf.L - 1].ptr : nullptr, cf.prec == OCCU_BF16 ? 1 : 0, csr.in_ptr,
      cf.aggr == OCCU_AGGR_MEAN, cf.slope,
      w.dh.as<float>(), (tcb && use_bits && ctx->hbits_layers >= cf.L)
                            ? reinterpret_cast<const uint32_t *>(w.hbits[cf.L - 1].ptr) : nullptr);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 3;
}

template <int D>
static int backward_layer_impl(occu_ctx *ctx, const DevCsr &csr, const BwdLayerArgs &a,
                               cudaStream_t st) {
  const occu_config &cf = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  Workspace &w = ctx->ws;
  const int i = a.layer;
  const float *P = ctx->params.as<float>();
  float *G = ctx->grads.as<float>();
  const int sms = ctx->num_sms;
  int n = 0;
  float *de = w.deA.as<float>();
  const bool tc = ctx->path != 1 && tc_supported(cf);
  const bool bf = a.bf;                     // OCCU_BF16: stored activations are BF16 (R28)
  const bool in_bf = bf && i > 0;           // h_in, e_in of layer 1 are the FP32 inputs
  if ((bf || cf.msg == OCCU_MSG_NEIGHBOR_SOFTMAX) && !(tc && a.g)) return -int(cudaErrorInvalidValue);
  int r;
  if (w.partial.ensure(3 * WG_SLOT_FLOATS * 4) != cudaSuccess) return -int(cudaErrorMemoryAllocation);
  float *slot = w.partial.as<float>();
  static const bool fuse_we = !getenv("OCCU_NO_FUSE_WE");   // A/B switch: dW_e in the layer-1 edge backward
  static const bool use_bits = !getenv("OCCU_NO_HBITS");     // A/B switch: LReLU'(h_in) from the sign bits
  // row scale exponents of DV, DZ, dP handed from their producers to the row-GEMMs that read
  // them (the same exponents the converters would compute: bitwise-neutral, A/B OCCU_NO_REXP)
  static const bool use_rexp = !getenv("OCCU_NO_REXP");
  int *dv_rexp = nullptr, *dz_rexp = nullptr, *dp_rexp = nullptr;
  if (use_rexp && tc) {
    if (w.rexp.ensure((2 * size_t(csr.E) + size_t(csr.N) + 4) * 4) != cudaSuccess) return -int(cudaErrorMemoryAllocation);
    dv_rexp = w.rexp.as<int>();
    dz_rexp = dv_rexp + csr.E;
    dp_rexp = dz_rexp + csr.E;
  }
  int *dv_used = nullptr, *dz_used = nullptr;   // exponents actually written this layer
  int we_blocks = 0;                        // > 0: dW_e partials already written by edge_bwd_small
  // the streaming gate backward (saved gates) leaves MG = dA[t] ⊙ g to the node backward
  const bool mg_from_g = tc && a.g && !getenv("OCCU_NODE_BWD_V1");
  float *MGo = mg_from_g ? nullptr : w.MG.as<float>();
  if (tc && csr.E > 0) {
    // a10: softmax / message backward (streaming with the saved gates, else g recomputed on
    // tensor cores), W_mᵀ dv, z recompute + σ', W_eᵀ dz on tensor cores
    if (a.g && cf.msg == OCCU_MSG_NEIGHBOR_SOFTMAX) {
      OCCU_PROF_BEGIN(ctx, "gate_bwd", st);
      gate_bwd_stream_kernel<D, false, true><<<grid_for((long(csr.E) + 31) / 32, NT / 32, 8 * sms), NT, 0, st>>>(
          a.g, a.dh, a.hbar, csr.in_src, csr.in_dst, csr.E, MGo, w.DV.as<float>(),
          a.h, csr.in_ptr, cf.aggr == OCCU_AGGR_MEAN, cf.slope);
      OCCU_PROF_END(ctx);
      LAUNCH_CHECK();
      ++n;
    } else if (a.g) {
      OCCU_PROF_BEGIN(ctx, "gate_bwd", st);
      dv_used = dv_rexp;
      if (bf)
        gate_bwd_stream_kernel<D, true><<<grid_for((long(csr.E) + 31) / 32, NT / 32, 8 * sms), NT, 0, st>>>(
            a.g, a.dh, a.hbar, csr.in_src, csr.in_dst, csr.E, MGo, w.DV.as<float>(), nullptr, nullptr, 0,
            0.01f, dv_rexp);
      else
        gate_bwd_stream_kernel<D, false><<<grid_for((long(csr.E) + 31) / 32, NT / 32, 8 * sms), NT, 0, st>>>(
            a.g, a.dh, a.hbar, csr.in_src, csr.in_dst, csr.E, MGo, w.DV.as<float>(), nullptr, nullptr, 0,
            0.01f, dv_rexp);
      OCCU_PROF_END(ctx);
      LAUNCH_CHECK();
      ++n;
    } else {
      if ((r = launch_bwd_gate_tc(ctx, csr, i, a.e, a.dh, nullptr, a.hbar, w.MG.as<float>(),
                                  w.DV.as<float>(), st)) < 0) return r;
      n += r;
    }
    if ((r = launch_plain_tc(ctx, w.DV.as<float>(), D, csr.E, 3, i, a.de_out, de,
                             "de_tc", st, nullptr, nullptr, false, nullptr, dv_used)) < 0) return r;
    n += r;
    if (a.Ke > 16 && bf) {
      if ((r = launch_bwd_edge_bf16(ctx, csr, i, a.e_in, a.Ke, a.e, de, a.p, a.q,
                                    w.DZ.as<float>(), w.dalpha.as<float>(), st)) < 0) return r;
      n += r;
    } else if (a.Ke > 16) {
      if ((r = launch_bwd_edge_tc(ctx, csr, i, a.e_in, a.Ke, a.e, de, a.p, a.q,
                                  w.DZ.as<float>(), w.dalpha.as<float>(), st, dz_rexp)) < 0) return r;
      dz_used = dz_rexp;
      n += r;
    } else {
      const int tiles = (csr.E + BM - 1) / BM;
      const int KS = a.Ke > D ? a.Ke : D;
      const size_t smB = (size_t(a.Ke) * D + BM * (KS + 4) + BM) * 4;
      (void)tiles;
      (void)smB;
      // layer 1 only (Ke <= 16): e_in is the FP32 e0; e' is BF16 in OCCU_BF16
      OCCU_PROF_BEGIN(ctx, "edge_bwd_e", st);
      const int eg = grid_for((long(csr.E) + 31) / 32, NT / 32, 8 * sms);
#define OCCU_EBS_ARGS a.e_in, a.Ke, a.e, de, P + L.W_e[i], a.p, a.q, csr.in_src, csr.in_dst, csr.E, \
    w.DZ.as<float>(), w.dalpha.as<float>()
      if (a.Ke == 4 && fuse_we) {
        // layer 1 with F_e = 4: dW_e accumulated here (per-block partials in the W_e slot); one
        // wave of resident blocks (each reduces its partial once) instead of several
        static const bool eb_cpa = !getenv("OCCU_EB_NOCPA");   // A/B switch (bitwise-equal results)
        const int egw = grid_for((long(csr.E) + 31) / 32, NT / 32, (eb_cpa ? 3 : 2) * sms);
        const size_t ebs = size_t(NT / 32) * EB_RING * (bf ? eb_slot_bytes<D, true>() : eb_slot_bytes<D, false>());
        if (eb_cpa && bf) {
          set_smem(edge_bwd_small_kernel<D, 4, true, true, true>, ebs);
          edge_bwd_small_kernel<D, 4, true, true, true><<<egw, NT, ebs, st>>>(OCCU_EBS_ARGS, slot + WG_SLOT_FLOATS);
        } else if (eb_cpa) {
          set_smem(edge_bwd_small_kernel<D, 4, false, true, true>, ebs);
          edge_bwd_small_kernel<D, 4, false, true, true><<<egw, NT, ebs, st>>>(OCCU_EBS_ARGS, slot + WG_SLOT_FLOATS);
        } else if (bf) {
          edge_bwd_small_kernel<D, 4, true, true><<<egw, NT, 0, st>>>(OCCU_EBS_ARGS, slot + WG_SLOT_FLOATS);
        } else {
          edge_bwd_small_kernel<D, 4, false, true><<<egw, NT, 0, st>>>(OCCU_EBS_ARGS, slot + WG_SLOT_FLOATS);
        }
        we_blocks = egw;
      } else if (a.Ke <= 4) {
        if (bf) edge_bwd_small_kernel<D, 4, true><<<eg, NT, 0, st>>>(OCCU_EBS_ARGS);
        else edge_bwd_small_kernel<D, 4, false><<<eg, NT, 0, st>>>(OCCU_EBS_ARGS);
      } else {
        if (bf) edge_bwd_small_kernel<D, 16, true><<<eg, NT, 0, st>>>(OCCU_EBS_ARGS);
        else edge_bwd_small_kernel<D, 16, false><<<eg, NT, 0, st>>>(OCCU_EBS_ARGS);
      }
#undef OCCU_EBS_ARGS
      OCCU_PROF_END(ctx);
      LAUNCH_CHECK();
      ++n;
    }
    if (a.de_prev) {
      if ((r = launch_plain_tc(ctx, w.DZ.as<float>(), D, csr.E, 4, i, nullptr,
                               a.de_prev, "de_prev_tc", st, nullptr, nullptr, false, nullptr, dz_used)) < 0) return r;
      n += r;
    }
  } else if (csr.E > 0) {
    const size_t smA = (2 * D * D + BM * (D + 4)) * 4 + 2 * BM * 4;
    set_smem(edge_bwd_m_kernel<D>, smA);
    const int tiles = (csr.E + BM - 1) / BM;
    OCCU_PROF_BEGIN(ctx, "edge_bwd_m", st);
    edge_bwd_m_kernel<D><<<grid_for(tiles, 1, sms), NT, smA, st>>>(
        a.e, P + L.W_m[i], a.hbar, a.h, a.dh, a.de_out, csr.in_src, csr.in_dst, csr.in_ptr, csr.E,
        cf.aggr == OCCU_AGGR_MEAN, cf.slope, w.MG.as<float>(), w.DV.as<float>(), de);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    ++n;
    const int KS = a.Ke > D ? a.Ke : D;
    const size_t smB = (size_t(a.Ke) * D + (a.de_prev ? D * a.Ke : 0) + BM * (KS + 4) + BM) * 4;
    set_smem(edge_bwd_e_kernel<D, false>, smB);
    OCCU_PROF_BEGIN(ctx, "edge_bwd_e", st);
    edge_bwd_e_kernel<D, false><<<grid_for(tiles, 1, sms), NT, smB, st>>>(
        a.e_in, a.Ke, a.e, de, P + L.W_e[i], a.p, a.q, csr.in_src, csr.in_dst, csr.E,
        w.DZ.as<float>(), w.dalpha.as<float>(), a.de_prev);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    ++n;
  }
  const int nb_blocks = grid_for(long(csr.N) * 32, NT, 16 * sms);
  // [da_s; da_d] partials from node_bwd on both kernel paths (float64 per block)
  if (w.dpart.ensure(size_t(nb_blocks) * 2 * D * 4) != cudaSuccess) return -int(cudaErrorMemoryAllocation);
  float *da_part = w.dpart.as<float>();
  OCCU_PROF_BEGIN(ctx, "node_bwd", st);
  static const int nbv = getenv("OCCU_NODE_BWD_V1") ? 0 : 1;     // A/B switch: 1 = v2 (default)
  const bool fromg = nbv && mg_from_g;
#define OCCU_NB_ARGS w.MG.as<float>(), w.dalpha.as<float>(), a.hbar, P + L.a_s[i], P + L.a_d[i], csr.out_ptr, \
    csr.out_pos, csr.in_ptr, csr.N, cf.slope, w.dP.as<float>(), w.dpq.as<float>(), da_part
  static const bool nb_cpa = !getenv("OCCU_NB_NOCPA");      // A/B switch (bitwise-equal results)
  const size_t nb_smem = size_t(NT / 32) * NB_RING * (bf ? nb_slot_bytes<D, true>() : nb_slot_bytes<D, false>());
  if (fromg && bf && nb_cpa) {
    set_smem(node_bwd_v2_kernel<D, true, true, true>, nb_smem);
    node_bwd_v2_kernel<D, true, true, true><<<nb_blocks, NT, nb_smem, st>>>(OCCU_NB_ARGS, a.g, a.dh, csr.in_dst, dp_rexp);
  } else if (fromg && nb_cpa) {
    set_smem(node_bwd_v2_kernel<D, false, true, true>, nb_smem);
    node_bwd_v2_kernel<D, false, true, true><<<nb_blocks, NT, nb_smem, st>>>(OCCU_NB_ARGS, a.g, a.dh, csr.in_dst, dp_rexp);
  } else if (fromg && bf)
    node_bwd_v2_kernel<D, true, true><<<nb_blocks, NT, 0, st>>>(OCCU_NB_ARGS, a.g, a.dh, csr.in_dst, dp_rexp);
  else if (fromg)
    node_bwd_v2_kernel<D, false, true><<<nb_blocks, NT, 0, st>>>(OCCU_NB_ARGS, a.g, a.dh, csr.in_dst, dp_rexp);
  else if (nbv && bf)
    node_bwd_v2_kernel<D, true, false><<<nb_blocks, NT, 0, st>>>(OCCU_NB_ARGS, nullptr, nullptr, nullptr, dp_rexp);
  else if (nbv)
    node_bwd_v2_kernel<D, false, false><<<nb_blocks, NT, 0, st>>>(OCCU_NB_ARGS, nullptr, nullptr, nullptr, dp_rexp);
  else if (bf)
    node_bwd_kernel<D, true><<<nb_blocks, NT, 0, st>>>(OCCU_NB_ARGS);
  else
    node_bwd_kernel<D, false><<<nb_blocks, NT, 0, st>>>(OCCU_NB_ARGS);
#undef OCCU_NB_ARGS
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  ++n;
  // dW_m = DVᵀ E' ; dW_e = DZᵀ E_in ; dW_u = dPᵀ H_in ; [da_s; da_d] = [dp dq]ᵀ h̄ — partial
  // sums into per-GEMM slots, all of the layer's split reductions in one launch
  ReduceJobs rj{};
  rj.j[rj.count++] = ReduceJob{da_part, G + L.a_s[i], long(2 * D), nb_blocks};
  if ((r = wgrad_deferred(ctx, w.DV.as<float>(), D, a.e, D, csr.E, G + L.W_m[i], st, bf, rj, slot)) < 0) return r;
  n += r;
  if (we_blocks > 0) {
    rj.j[rj.count++] = ReduceJob{slot + WG_SLOT_FLOATS, G + L.W_e[i], long(D) * a.Ke, we_blocks};
  } else {
    if ((r = wgrad_deferred(ctx, w.DZ.as<float>(), D, a.e_in, a.Ke, csr.E, G + L.W_e[i], st, in_bf, rj,
                            slot + WG_SLOT_FLOATS)) < 0) return r;
    n += r;
  }
  if ((r = wgrad_deferred(ctx, w.dP.as<float>(), D, a.h_in, a.K, csr.N, G + L.W_u[i], st, in_bf, rj,
                          slot + 2 * WG_SLOT_FLOATS)) < 0) return r;
  n += r;
  if ((r = launch_multi_reduce(ctx, rj, st)) < 0) return r;
  n += r;
  if (a.dh_prev && csr.N > 0 && tc) {   // dh^{i-1} = dP W_u on tensor cores
    if ((r = launch_plain_tc(ctx, w.dP.as<float>(), D, csr.N, 5, i, nullptr, a.dh_prev,
                             "dh_prev_tc", st, a.h_in, csr.in_ptr, in_bf,
                             use_bits ? a.h_in_bits : nullptr, nbv ? dp_rexp : nullptr)) < 0) return r;
    n += r;
  } else if (a.dh_prev && csr.N > 0) {   // dh^{i-1} = dP W_u  (K == D for i > 0)
    const size_t sm1 = (size_t(D) * D + BM * (D + 4)) * 4;
    set_smem(node_gemm_kernel<D, 1>, sm1);
    const int tiles = (csr.N + BM - 1) / BM;
    OCCU_PROF_BEGIN(ctx, "dh_prev_gemm", st);
    node_gemm_kernel<D, 1><<<grid_for(tiles, 1, 2 * sms), NT, sm1, st>>>(
        w.dP.as<float>(), D, P + L.W_u[i], nullptr, nullptr, csr.N, cf.slope, a.dh_prev,
        nullptr, nullptr);
    OCCU_PROF_END(ctx);
    LAUNCH_CHECK();
    ++n;
  }
  return n;
}

int launch_backward_layer(occu_ctx *ctx, const DevCsr &csr, const BwdLayerArgs &a,
                          cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return backward_layer_impl<64>(ctx, csr, a, st);
    case 128: return backward_layer_impl<128>(ctx, csr, a, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

int launch_adam(occu_ctx *ctx, float lr, cudaStream_t st) {
  ctx->params_version += 1;        // tensor-core weight images must be rebuilt
  const long n = long(ctx->layout.total);
  const double b1 = 0.9, b2 = 0.999;
  const double bc1 = 1.0 - pow(b1, double(ctx->adam_t));
  const double bc2 = 1.0 - pow(b2, double(ctx->adam_t));
  OCCU_PROF_BEGIN(ctx, "adam", st);
  adam_kernel<<<grid_for(n, 256, 1024), 256, 0, st>>>(
      ctx->params.as<float>(), ctx->grads.as<float>(), ctx->adam_m.as<float>(),
      ctx->adam_v.as<float>(), n, lr, ctx->weight_decay, float(b1), float(b2), float(bc1),
      float(bc2), 1e-8f);
  OCCU_PROF_END(ctx);
  LAUNCH_CHECK();
  return 1;
}

}  // namespace occu
