// NEXT-3: Graphormer layers (P153-P157; R35-R37), per graph over its
// node set, between the last ANEE round and the readout:
//   h̄ = MHA(LN(h)) + h,     h' = FFN(LN(h̄)) + h̄
// MHA = self-attention over the nodes of the node's own graph (block-diagonal over the batch).
//
// B200 mapping (OCCU_FP32):
//  * the six d x d projections (W_q, W_k, W_v, W_o, FFN W1, W2) are tensor-core row-GEMMs
//    (tcgen05 fp16x2 split, bias / ReLU / residual-add epilogues: launch_bias_tc,
//    launch_bias_add_tc);
//  * LayerNorm: warp per row, FP32, two passes over the row in registers;
//  * attention (gph_attn_kernel): the only contraction that grows with n², flash-style:
//    CTA = 64 query rows x one head, 4 warps x 16 rows; the keys / values of the rows'
//    graphs stream through shared memory in 64-row blocks (cp.async, double-buffered); scores
//    and P·V on tensor cores with mma.sync m16n8k8 TF32 in the 3-product split (x = hi + lo,
//    hi·hi + hi·lo + lo·hi, ~2^-22 relative: the FP32 tolerance of north_star), online
//    softmax in registers (ex2 with log2(e)/√d_h folded into Q).  A query tile may straddle
//    graphs: the key range is the union of its rows' graphs and every score outside the
//    row's own graph is masked, so no host-side tile list is needed.
//    P's accumulator fragment feeds the P·V MMA without shuffles: inside each 8-key group the
//    k order of the P·V product is permuted (k = t <-> key 2t, k = t + 4 <-> key 2t + 1) and
//    the V fragment is read in the same order.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdlib.h>
#include <stdint.h>

#include "occu_internal.h"
#include "tc_common.cuh"

namespace occu {
namespace {

constexpr float L2E = 1.4426950408889634f;
constexpr int QT = 64;     // query rows per CTA
constexpr int KT = 64;     // keys per shared-memory block
constexpr int AW = 4;      // warps per CTA

__device__ __forceinline__ float ex2f(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// x = hi + lo, hi = x rounded to tf32 (the MMA reads hi exactly; lo is truncated to tf32 by the
// MMA, an error of 2^-11·|lo| <= 2^-22·|x|).
__device__ __forceinline__ void split_tf32(float x, uint32_t &hi, uint32_t &lo) {
  uint32_t h;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(h) : "f"(x));
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

// c += (ah + al)(bh + bl) without the al·bl term; small products first
__device__ __forceinline__ void mma3(float (&c)[4], const uint32_t (&ah)[4], const uint32_t (&al)[4],
                                     uint32_t bh0, uint32_t bh1, uint32_t bl0, uint32_t bl1) {
  mma_tf32(c, al, bh0, bh1);
  mma_tf32(c, ah, bl0, bl1);
  mma_tf32(c, ah, bh0, bh1);
}

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, bool pred) {
  const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "r"(pred ? 16 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// Y[r] = LN(X[r]) · g + b over D channels (eps 1e-5, biased variance); warp per row.
template <int D>
__global__ void __launch_bounds__(256) gph_ln_kernel(const float *__restrict__ X, int N,
                                                     const float *__restrict__ g,
                                                     const float *__restrict__ b,
                                                     float *__restrict__ Y) {
  constexpr int V = D / 128;              // float4 per lane
  pdl_trigger();
  const int lane = threadIdx.x & 31;
  const long row = long(blockIdx.x) * 8 + (threadIdx.x >> 5);
  if (row >= N) return;
  float4 x[V];
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < V; ++i) {
    x[i] = __ldg(reinterpret_cast<const float4 *>(X + row * D) + lane + 32 * i);
    s += (x[i].x + x[i].y) + (x[i].z + x[i].w);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mu = s * (1.f / float(D));
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < V; ++i) {
    const float a0 = x[i].x - mu, a1 = x[i].y - mu, a2 = x[i].z - mu, a3 = x[i].w - mu;
    q = fmaf(a0, a0, fmaf(a1, a1, fmaf(a2, a2, fmaf(a3, a3, q))));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
  const float inv = rsqrtf(q * (1.f / float(D)) + 1e-5f);
#pragma unroll
  for (int i = 0; i < V; ++i) {
    const int c = (lane + 32 * i) * 4;
    const float4 gg = __ldg(reinterpret_cast<const float4 *>(g + c));
    const float4 bb = __ldg(reinterpret_cast<const float4 *>(b + c));
    float4 y;
    y.x = (x[i].x - mu) * inv * gg.x + bb.x;
    y.y = (x[i].y - mu) * inv * gg.y + bb.y;
    y.z = (x[i].z - mu) * inv * gg.z + bb.z;
    y.w = (x[i].w - mu) * inv * gg.w + bb.w;
    reinterpret_cast<float4 *>(Y + row * D)[lane + 32 * i] = y;
  }
}

// D = 64 variant of the LN (float2 per lane)
template <>
__global__ void __launch_bounds__(256) gph_ln_kernel<64>(const float *__restrict__ X, int N,
                                                         const float *__restrict__ g,
                                                         const float *__restrict__ b,
                                                         float *__restrict__ Y) {
  pdl_trigger();
  const int lane = threadIdx.x & 31;
  const long row = long(blockIdx.x) * 8 + (threadIdx.x >> 5);
  if (row >= N) return;
  const float2 x = __ldg(reinterpret_cast<const float2 *>(X + row * 64) + lane);
  float s = x.x + x.y;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mu = s * (1.f / 64.f);
  const float a0 = x.x - mu, a1 = x.y - mu;
  float q = fmaf(a0, a0, a1 * a1);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
  const float inv = rsqrtf(q * (1.f / 64.f) + 1e-5f);
  const float2 gg = __ldg(reinterpret_cast<const float2 *>(g) + lane);
  const float2 bb = __ldg(reinterpret_cast<const float2 *>(b) + lane);
  reinterpret_cast<float2 *>(Y + row * 64)[lane] = make_float2(a0 * inv * gg.x + bb.x, a1 * inv * gg.y + bb.y);
}

struct AttnArgs {
  const float *Q, *K, *V;        // [N][D] each (head h = columns h·DH .. h·DH + DH - 1)
  const int32_t *node_off;       // [B+1]
  const int32_t *node_graph;     // [N]
  float *O;                      // [N][D]
  int N, D;
  float qscale;                  // log2(e) / sqrt(DH)
};

// Flash attention over each row's own graph; grid (ceil(N / 64), heads), 128 threads.
template <int DH>
__global__ void __launch_bounds__(AW * 32) gph_attn_kernel(const AttnArgs a) {
  constexpr int KS = DH / 8;            // k-steps of Q·Kᵀ
  constexpr int NO = DH / 8;            // n-tiles of the output
  constexpr int SP = DH + 4;            // smem row stride (floats): conflict-free fragment reads
  extern __shared__ float4 attn_smem[];                  // K [2][KT][SP], V [2][KT][SP]
  float *const Ks0 = reinterpret_cast<float *>(attn_smem);
  float *const Vs0 = Ks0 + 2 * KT * SP;
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, t = lane & 3;
  const int head = blockIdx.y;
  const long q0 = long(blockIdx.x) * QT;
  const int D = a.D;
  const long hc = long(head) * DH;

  // key range of the CTA: union of its rows' graphs
  const long qlast = min(q0 + QT, long(a.N)) - 1;
  const int kbeg = __ldg(a.node_off + __ldg(a.node_graph + q0));
  const int kend = __ldg(a.node_off + __ldg(a.node_graph + qlast) + 1);

  // this thread's two rows and their graphs' key ranges
  const long ra = q0 + warp * 16 + g, rb = ra + 8;
  int loa = 0, hia = 0, lob = 0, hib = 0;
  if (ra < a.N) { const int gr = __ldg(a.node_graph + ra); loa = __ldg(a.node_off + gr); hia = __ldg(a.node_off + gr + 1); }
  if (rb < a.N) { const int gr = __ldg(a.node_graph + rb); lob = __ldg(a.node_off + gr); hib = __ldg(a.node_off + gr + 1); }
  // warp key range (blocks outside it are skipped by this warp)
  int wlo = min(ra < a.N ? loa : INT32_MAX, rb < a.N ? lob : INT32_MAX);
  int whi = max(hia, hib);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    wlo = min(wlo, __shfl_xor_sync(0xffffffffu, wlo, o));
    whi = max(whi, __shfl_xor_sync(0xffffffffu, whi, o));
  }

  // Q fragments (scaled, split), rows ra / rb, dims ks·8 + t (+4)
  uint32_t qh[KS][4], ql[KS][4];
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
    const int c = ks * 8 + t;
    const float x0 = ra < a.N ? __ldg(a.Q + ra * D + hc + c) * a.qscale : 0.f;
    const float x1 = rb < a.N ? __ldg(a.Q + rb * D + hc + c) * a.qscale : 0.f;
    const float x2 = ra < a.N ? __ldg(a.Q + ra * D + hc + c + 4) * a.qscale : 0.f;
    const float x3 = rb < a.N ? __ldg(a.Q + rb * D + hc + c + 4) * a.qscale : 0.f;
    split_tf32(x0, qh[ks][0], ql[ks][0]);
    split_tf32(x1, qh[ks][1], ql[ks][1]);
    split_tf32(x2, qh[ks][2], ql[ks][2]);
    split_tf32(x3, qh[ks][3], ql[ks][3]);
  }

  float o[NO][4];
#pragma unroll
  for (int n = 0; n < NO; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
  float ma = -INFINITY, mb = -INFINITY, la = 0.f, lb = 0.f;

  // stage one 64-key block of K and V (rows beyond kend zero-filled)
  auto stage = [&](int buf, int kb) {
    constexpr int C4 = DH / 4;                  // 16-byte chunks per row
    for (int i = threadIdx.x; i < KT * C4; i += AW * 32) {
      const int r = i / C4, c = (i % C4) * 4;
      const long key = long(kb) + r;
      const bool ok = key < kend;
      const long src = (ok ? key : kbeg) * D + hc + c;
      cp_async16(Ks0 + (buf * KT + r) * SP + c, a.K + src, ok);
      cp_async16(Vs0 + (buf * KT + r) * SP + c, a.V + src, ok);
    }
    cp_async_commit();
  };

  const int nblk = (kend - kbeg + KT - 1) / KT;
  if (nblk > 0) stage(0, kbeg);
  for (int bi = 0; bi < nblk; ++bi) {
    const int kb = kbeg + bi * KT;
    if (bi + 1 < nblk) {
      stage((bi + 1) & 1, kb + KT);
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    const float *Kb = Ks0 + (bi & 1) * KT * SP, *Vb = Vs0 + (bi & 1) * KT * SP;
    if (kb < whi && kb + KT > wlo) {
      // ---- S = Q Kᵀ (16 x 64 per warp), already in the log2 domain
      float s[8][4];
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        s[nt][0] = s[nt][1] = s[nt][2] = s[nt][3] = 0.f;
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
          const float *kr = Kb + (nt * 8 + g) * SP + ks * 8 + t;
          uint32_t bh0, bl0, bh1, bl1;
          split_tf32(kr[0], bh0, bl0);
          split_tf32(kr[4], bh1, bl1);
          mma3(s[nt], qh[ks], ql[ks], bh0, bh1, bl0, bl1);
        }
      }
      // ---- mask keys outside each row's graph, online softmax
      float bma = -INFINITY, bmb = -INFINITY;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const int k0 = kb + nt * 8 + 2 * t;
        if (!(k0 >= loa && k0 < hia)) s[nt][0] = -INFINITY;
        if (!(k0 + 1 >= loa && k0 + 1 < hia)) s[nt][1] = -INFINITY;
        if (!(k0 >= lob && k0 < hib)) s[nt][2] = -INFINITY;
        if (!(k0 + 1 >= lob && k0 + 1 < hib)) s[nt][3] = -INFINITY;
        bma = fmaxf(bma, fmaxf(s[nt][0], s[nt][1]));
        bmb = fmaxf(bmb, fmaxf(s[nt][2], s[nt][3]));
      }
#pragma unroll
      for (int o2 = 1; o2 <= 2; o2 <<= 1) {
        bma = fmaxf(bma, __shfl_xor_sync(0xffffffffu, bma, o2));
        bmb = fmaxf(bmb, __shfl_xor_sync(0xffffffffu, bmb, o2));
      }
      const float mna = fmaxf(ma, bma), mnb = fmaxf(mb, bmb);
      const float refa = mna == -INFINITY ? 0.f : mna, refb = mnb == -INFINITY ? 0.f : mnb;
      const float fa = ex2f(ma - refa), fb = ex2f(mb - refb);     // 0 while m = -inf
      ma = mna; mb = mnb;
      float sa = 0.f, sb = 0.f;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        s[nt][0] = ex2f(s[nt][0] - refa); s[nt][1] = ex2f(s[nt][1] - refa);
        s[nt][2] = ex2f(s[nt][2] - refb); s[nt][3] = ex2f(s[nt][3] - refb);
        sa += s[nt][0] + s[nt][1];
        sb += s[nt][2] + s[nt][3];
      }
      la = la * fa + sa;          // per-thread partial sums (quad-reduced at the end)
      lb = lb * fb + sb;
#pragma unroll
      for (int n = 0; n < NO; ++n) {
        o[n][0] *= fa; o[n][1] *= fa; o[n][2] *= fb; o[n][3] *= fb;
      }
      // ---- O += P V: k-group j = the 8 keys of score tile j, k order permuted (see top)
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        uint32_t ph[4], pl[4];
        split_tf32(s[j][0], ph[0], pl[0]);     // (row g,     k = t)     <- key 2t
        split_tf32(s[j][2], ph[1], pl[1]);     // (row g + 8, k = t)     <- key 2t
        split_tf32(s[j][1], ph[2], pl[2]);     // (row g,     k = t + 4) <- key 2t + 1
        split_tf32(s[j][3], ph[3], pl[3]);     // (row g + 8, k = t + 4) <- key 2t + 1
        const float *v0 = Vb + (j * 8 + 2 * t) * SP + g;
#pragma unroll
        for (int n = 0; n < NO; ++n) {
          uint32_t bh0, bl0, bh1, bl1;
          split_tf32(v0[n * 8], bh0, bl0);          // V[key 2t][n·8 + g]
          split_tf32(v0[SP + n * 8], bh1, bl1);     // V[key 2t + 1][n·8 + g]
          mma3(o[n], ph, pl, bh0, bh1, bl0, bl1);
        }
      }
    }
    __syncthreads();              // the buffer is restaged next iteration
  }
  // quad-reduce the row sums, normalise, store rows ra / rb (float2 per n-tile)
#pragma unroll
  for (int o2 = 1; o2 <= 2; o2 <<= 1) {
    la += __shfl_xor_sync(0xffffffffu, la, o2);
    lb += __shfl_xor_sync(0xffffffffu, lb, o2);
  }
  const float ia = la > 0.f ? 1.f / la : 0.f, ib = lb > 0.f ? 1.f / lb : 0.f;
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const long c = hc + n * 8 + 2 * t;
    if (ra < a.N) *reinterpret_cast<float2 *>(a.O + ra * D + c) = make_float2(o[n][0] * ia, o[n][1] * ia);
    if (rb < a.N) *reinterpret_cast<float2 *>(a.O + rb * D + c) = make_float2(o[n][2] * ib, o[n][3] * ib);
  }
}

// ---- FP16 variant: mma.sync m16n8k16 with the fp16x2 split (x = hi + lo, both fp16;
// hi·hi + hi·lo + lo·hi), half the MMA instructions of the TF32 split for the same products.
// K / V blocks land by cp.async as FP32 and are split once per CTA into fp16 hi / lo tiles
// [key][DH + 8] that every warp reads with ldmatrix (V with .trans for the P·V operand).
// FP16 operand range: |Q·log2(e)/√d_h|, |K|, |V| < 65504 (LayerNorm inputs keep them O(10));
// values below 2^-14 lose relative precision in the lo part, an absolute error < 2^-24.
__device__ __forceinline__ void mma_f16(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ void split_h2(float x0, float x1, uint32_t &hi, uint32_t &lo) {
  const __half2 h = __floats2half2_rn(x0, x1);
  const float2 hf = __half22float2(h);
  const __half2 l = __floats2half2_rn(x0 - hf.x, x1 - hf.y);
  hi = *reinterpret_cast<const uint32_t *>(&h);
  lo = *reinterpret_cast<const uint32_t *>(&l);
}
__device__ __forceinline__ uint32_t pack_h2(float x0, float x1) {
  const __half2 h = __floats2half2_rn(x0, x1);
  return *reinterpret_cast<const uint32_t *>(&h);
}
__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}

template <int DH>
struct F16Smem {
  static constexpr int SF = DH + 4;        // fp32 staging row stride (floats)
  static constexpr int SH = DH + 8;        // fp16 tile row stride (halves): 16-byte rows, ldmatrix conflict-free
  static constexpr size_t stage_floats = size_t(2) * 2 * KT * SF;     // [buf][K|V][KT][SF]
  static constexpr size_t tile_halves = size_t(4) * KT * SH;          // Kh, Kl, Vh, Vl
  static constexpr size_t bytes = stage_floats * 4 + tile_halves * 2;
};

template <int DH>
__global__ void __launch_bounds__(AW * 32) gph_attn_f16_kernel(const AttnArgs a) {
  using S = F16Smem<DH>;
  constexpr int SF = S::SF, SH = S::SH;
  constexpr int KS = DH / 16;           // k-steps of Q·Kᵀ
  constexpr int NO = DH / 8;            // output n-tiles
  extern __shared__ float4 attn_smem[];
  float *const stg = reinterpret_cast<float *>(attn_smem);                     // [2][2][KT][SF]
  __half *const tiles = reinterpret_cast<__half *>(stg + S::stage_floats);     // [4][KT][SH]
  __half *const Kh = tiles, *const Kl = tiles + KT * SH, *const Vh = tiles + 2 * KT * SH,
         *const Vl = tiles + 3 * KT * SH;
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, t = lane & 3;
  const long q0 = long(blockIdx.x) * QT;
  const int D = a.D;
  const long hc = long(blockIdx.y) * DH;

  const long qlast = min(q0 + QT, long(a.N)) - 1;
  const int kbeg = __ldg(a.node_off + __ldg(a.node_graph + q0));
  const int kend = __ldg(a.node_off + __ldg(a.node_graph + qlast) + 1);
  const long ra = q0 + warp * 16 + g, rb = ra + 8;
  int loa = 0, hia = 0, lob = 0, hib = 0;
  if (ra < a.N) { const int gr = __ldg(a.node_graph + ra); loa = __ldg(a.node_off + gr); hia = __ldg(a.node_off + gr + 1); }
  if (rb < a.N) { const int gr = __ldg(a.node_graph + rb); lob = __ldg(a.node_off + gr); hib = __ldg(a.node_off + gr + 1); }
  int wlo = min(ra < a.N ? loa : INT32_MAX, rb < a.N ? lob : INT32_MAX);
  int whi = max(hia, hib);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    wlo = min(wlo, __shfl_xor_sync(0xffffffffu, wlo, o));
    whi = max(whi, __shfl_xor_sync(0xffffffffu, whi, o));
  }

  // Q fragments (scaled, fp16x2 split): a0a1 (g, 2t), a2a3 (g+8, 2t), a4a5 (g, 2t+8), a6a7 (g+8, 2t+8)
  uint32_t qh[KS][4], ql[KS][4];
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const long r = (q & 1) ? rb : ra;
      const int c = ks * 16 + (q >> 1) * 8 + 2 * t;
      float2 x = make_float2(0.f, 0.f);
      if (r < a.N) x = __ldg(reinterpret_cast<const float2 *>(a.Q + r * D + hc + c));
      split_h2(x.x * a.qscale, x.y * a.qscale, qh[ks][q], ql[ks][q]);
    }
  }

  float o[NO][4];
#pragma unroll
  for (int n = 0; n < NO; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
  float ma = -INFINITY, mb = -INFINITY, la = 0.f, lb = 0.f;

  auto stage = [&](int buf, int kb) {
    constexpr int C4 = DH / 4;
    float *Ks = stg + (buf * 2) * KT * SF, *Vs = stg + (buf * 2 + 1) * KT * SF;
    for (int i = threadIdx.x; i < KT * C4; i += AW * 32) {
      const int r = i / C4, c = (i % C4) * 4;
      const long key = long(kb) + r;
      const bool ok = key < kend;
      const long src = (ok ? key : kbeg) * D + hc + c;
      cp_async16(Ks + r * SF + c, a.K + src, ok);
      cp_async16(Vs + r * SF + c, a.V + src, ok);
    }
    cp_async_commit();
  };

  // ldmatrix row addresses (per thread, fixed): matrix q = lane >> 3, row lane & 7
  const int mq = lane >> 3, mr = lane & 7;
  const uint32_t kh_base = static_cast<uint32_t>(__cvta_generic_to_shared(Kh));
  const uint32_t kl_base = static_cast<uint32_t>(__cvta_generic_to_shared(Kl));
  const uint32_t vh_base = static_cast<uint32_t>(__cvta_generic_to_shared(Vh));
  const uint32_t vl_base = static_cast<uint32_t>(__cvta_generic_to_shared(Vl));
  // K (non-trans): matrices (nt + (q>>1), dims ks*16 + (q&1)*8): offset of row key (q>>1)*8 + mr
  const uint32_t koff = uint32_t((((mq >> 1) * 8 + mr) * SH + (mq & 1) * 8) * 2);
  // V (trans): matrices (keys 16kk + (q&1)*8 + mr, dims (n + (q>>1))*8)
  const uint32_t voff = uint32_t((((mq & 1) * 8 + mr) * SH + (mq >> 1) * 8) * 2);

  const int nblk = (kend - kbeg + KT - 1) / KT;
  if (nblk > 0) stage(0, kbeg);
  for (int bi = 0; bi < nblk; ++bi) {
    const int kb = kbeg + bi * KT;
    if (bi + 1 < nblk) {
      stage((bi + 1) & 1, kb + KT);
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    {   // split the FP32 block into the fp16 hi / lo tiles (once per CTA)
      const float *Ks = stg + ((bi & 1) * 2) * KT * SF, *Vs = stg + ((bi & 1) * 2 + 1) * KT * SF;
      constexpr int C4 = DH / 4;
      for (int i = threadIdx.x; i < KT * C4; i += AW * 32) {
        const int r = i / C4, c = (i % C4) * 4;
        const float4 kx = *reinterpret_cast<const float4 *>(Ks + r * SF + c);
        const float4 vx = *reinterpret_cast<const float4 *>(Vs + r * SF + c);
        uint32_t h0, l0, h1, l1;
        split_h2(kx.x, kx.y, h0, l0);
        split_h2(kx.z, kx.w, h1, l1);
        *reinterpret_cast<uint2 *>(Kh + r * SH + c) = make_uint2(h0, h1);
        *reinterpret_cast<uint2 *>(Kl + r * SH + c) = make_uint2(l0, l1);
        split_h2(vx.x, vx.y, h0, l0);
        split_h2(vx.z, vx.w, h1, l1);
        *reinterpret_cast<uint2 *>(Vh + r * SH + c) = make_uint2(h0, h1);
        *reinterpret_cast<uint2 *>(Vl + r * SH + c) = make_uint2(l0, l1);
      }
    }
    __syncthreads();
    if (kb < whi && kb + KT > wlo) {
      float s[8][4];
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) s[nt][0] = s[nt][1] = s[nt][2] = s[nt][3] = 0.f;
#pragma unroll
      for (int np = 0; np < 4; ++np) {          // n-tile pairs (2·np, 2·np + 1)
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
          const uint32_t off = koff + uint32_t((np * 16 * SH + ks * 16) * 2);
          uint32_t bh[4], bl[4];
          ldsm_x4(kh_base + off, bh);
          ldsm_x4(kl_base + off, bl);
          mma_f16(s[2 * np], ql[ks], bh[0], bh[1]);
          mma_f16(s[2 * np], qh[ks], bl[0], bl[1]);
          mma_f16(s[2 * np], qh[ks], bh[0], bh[1]);
          mma_f16(s[2 * np + 1], ql[ks], bh[2], bh[3]);
          mma_f16(s[2 * np + 1], qh[ks], bl[2], bl[3]);
          mma_f16(s[2 * np + 1], qh[ks], bh[2], bh[3]);
        }
      }
      float bma = -INFINITY, bmb = -INFINITY;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const int k0 = kb + nt * 8 + 2 * t;
        if (!(k0 >= loa && k0 < hia)) s[nt][0] = -INFINITY;
        if (!(k0 + 1 >= loa && k0 + 1 < hia)) s[nt][1] = -INFINITY;
        if (!(k0 >= lob && k0 < hib)) s[nt][2] = -INFINITY;
        if (!(k0 + 1 >= lob && k0 + 1 < hib)) s[nt][3] = -INFINITY;
        bma = fmaxf(bma, fmaxf(s[nt][0], s[nt][1]));
        bmb = fmaxf(bmb, fmaxf(s[nt][2], s[nt][3]));
      }
#pragma unroll
      for (int o2 = 1; o2 <= 2; o2 <<= 1) {
        bma = fmaxf(bma, __shfl_xor_sync(0xffffffffu, bma, o2));
        bmb = fmaxf(bmb, __shfl_xor_sync(0xffffffffu, bmb, o2));
      }
      const float mna = fmaxf(ma, bma), mnb = fmaxf(mb, bmb);
      const float refa = mna == -INFINITY ? 0.f : mna, refb = mnb == -INFINITY ? 0.f : mnb;
      const float fa = ex2f(ma - refa), fb = ex2f(mb - refb);
      ma = mna; mb = mnb;
      float sa = 0.f, sb = 0.f;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        s[nt][0] = ex2f(s[nt][0] - refa); s[nt][1] = ex2f(s[nt][1] - refa);
        s[nt][2] = ex2f(s[nt][2] - refb); s[nt][3] = ex2f(s[nt][3] - refb);
        sa += s[nt][0] + s[nt][1];
        sb += s[nt][2] + s[nt][3];
      }
      la = la * fa + sa;
      lb = lb * fb + sb;
#pragma unroll
      for (int n = 0; n < NO; ++n) {
        o[n][0] *= fa; o[n][1] *= fa; o[n][2] *= fb; o[n][3] *= fb;
      }
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {            // 16-key chunks
        uint32_t ph[4], pl[4];
        split_h2(s[2 * kk][0], s[2 * kk][1], ph[0], pl[0]);
        split_h2(s[2 * kk][2], s[2 * kk][3], ph[1], pl[1]);
        split_h2(s[2 * kk + 1][0], s[2 * kk + 1][1], ph[2], pl[2]);
        split_h2(s[2 * kk + 1][2], s[2 * kk + 1][3], ph[3], pl[3]);
#pragma unroll
        for (int np = 0; np < NO / 2; ++np) {     // output n-tile pairs
          const uint32_t off = voff + uint32_t((kk * 16 * SH + np * 16) * 2);
          uint32_t bh[4], bl[4];
          ldsm_x4_t(vh_base + off, bh);
          ldsm_x4_t(vl_base + off, bl);
          mma_f16(o[2 * np], pl, bh[0], bh[1]);
          mma_f16(o[2 * np], ph, bl[0], bl[1]);
          mma_f16(o[2 * np], ph, bh[0], bh[1]);
          mma_f16(o[2 * np + 1], pl, bh[2], bh[3]);
          mma_f16(o[2 * np + 1], ph, bl[2], bl[3]);
          mma_f16(o[2 * np + 1], ph, bh[2], bh[3]);
        }
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int o2 = 1; o2 <= 2; o2 <<= 1) {
    la += __shfl_xor_sync(0xffffffffu, la, o2);
    lb += __shfl_xor_sync(0xffffffffu, lb, o2);
  }
  const float ia = la > 0.f ? 1.f / la : 0.f, ib = lb > 0.f ? 1.f / lb : 0.f;
#pragma unroll
  for (int n = 0; n < NO; ++n) {
    const long c = hc + n * 8 + 2 * t;
    if (ra < a.N) *reinterpret_cast<float2 *>(a.O + ra * D + c) = make_float2(o[n][0] * ia, o[n][1] * ia);
    if (rb < a.N) *reinterpret_cast<float2 *>(a.O + rb * D + c) = make_float2(o[n][2] * ib, o[n][3] * ib);
  }
}

// ---- tcgen05 variant (d_h = 32): CTA = 128 query rows x one head, thread = query row = TMEM
// lane.  Q (scaled, fp16x2 split) lives in TMEM as the A operand; per 64-key block the CTA
// splits K into fp16 hi / lo SW128 tiles (B of S = Q·Kᵀ, N = 64) and V transposed into SW128
// tiles (B of O += P·V, N = 32, K = 64 keys); one thread issues 3 tcgen05.mma per K step for
// each product (hi·hi + hi·lo + lo·hi, FP32 accumulation in TMEM).  Each thread reads its
// row of S from TMEM (masking keys outside its graph), runs the online softmax, writes P hi / lo
// back to TMEM as the A operand of P·V and rescales its O row in TMEM.  Steps are serialised
// inside a CTA; two CTAs per SM (256 TMEM columns each) overlap one another.
namespace gtc {
constexpr int KB = 64;                       // keys per block
constexpr uint32_t TCOLS = 128;
// TMEM columns: Q hi / lo (16 each), S (64; P hi / lo overwrite it once the row is read), O (32)
constexpr uint32_t QH = 0, QL = 16, SC = 32, PH = 32, PL = 64, OC = 96;
constexpr uint32_t K_BYTES = KB * 128, V_BYTES = 32 * 128;
constexpr size_t SMEM = 50 * 1024;           // caps residency at four CTAs per SM (TMEM budget)
}

// spin (no back-off sleep): the waits here are short MMAs on the critical path
__device__ __forceinline__ void mbar_spin(uint64_t *bar, uint32_t parity) {
  const uint32_t a = tc::smem_u32(bar);
  while (!tc::mbar_try_wait(a, parity)) {
  }
}

__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// SPLIT = false (OCCU_BF16, R42): one fp16 product per step (Q, K, V, P rounded to fp16).
template <bool SPLIT>
__global__ void __launch_bounds__(128, 4) gph_attn_tc_kernel(const AttnArgs a) {
  using namespace gtc;
  extern __shared__ __align__(1024) uint8_t gsm_raw[];
  uint8_t *sm = gsm_raw + ((1024u - (tc::smem_u32(gsm_raw) & 1023u)) & 1023u);
  uint8_t *Kh = sm, *Kl = sm + K_BYTES, *Vh = sm + 2 * K_BYTES, *Vl = Vh + V_BYTES;
  uint64_t *bar = reinterpret_cast<uint64_t *>(Vl + V_BYTES);
  uint32_t *slot = reinterpret_cast<uint32_t *>(bar + 1);
  const int t = threadIdx.x, warp = t >> 5, lane = t & 31;
  const long q0 = long(blockIdx.x) * 128;
  const int D = a.D;
  const long hc = long(blockIdx.y) * 32;
  pdl_trigger();
  if (warp == 0) tc::tmem_alloc<TCOLS>(slot);
  if (t == 0) {
    tc::mbar_init(bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  const uint32_t tmem = *slot;
  const uint32_t lane_base = tmem + (uint32_t(warp * 32) << 16);

  const long r = q0 + t;
  const bool live = r < a.N;
  const long qlast = min(q0 + 128, long(a.N)) - 1;
  const int kbeg = __ldg(a.node_off + __ldg(a.node_graph + q0));
  const int kend = __ldg(a.node_off + __ldg(a.node_graph + qlast) + 1);
  int lo = 0, hi = 0;
  if (live) {
    const int gr = __ldg(a.node_graph + r);
    lo = __ldg(a.node_off + gr);
    hi = __ldg(a.node_off + gr + 1);
  }
  {   // Q row -> TMEM (scaled, fp16x2 split); O row = 0
    uint32_t qh[16], ql[16], z[32];
#pragma unroll
    for (int c = 0; c < 32; c += 4) {
      float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
      if (live) x = __ldg(reinterpret_cast<const float4 *>(a.Q + r * D + hc + c));
      split_h2(x.x * a.qscale, x.y * a.qscale, qh[c / 2], ql[c / 2]);
      split_h2(x.z * a.qscale, x.w * a.qscale, qh[c / 2 + 1], ql[c / 2 + 1]);
    }
#pragma unroll
    for (int c = 0; c < 32; ++c) z[c] = 0u;
    tc::tmem_st16(lane_base + QH, qh);
    tc::tmem_st16(lane_base + QL, ql);
    tc::tmem_st32(lane_base + OC, z);
    tc::tmem_st_wait();
  }
  const uint32_t kh_a = tc::smem_u32(Kh), kl_a = tc::smem_u32(Kl), vh_a = tc::smem_u32(Vh),
                 vl_a = tc::smem_u32(Vl);
  const uint32_t id_s = tc::idesc(128, KB, tc::FMT_F16), id_o = tc::idesc(128, 32, tc::FMT_F16);
  float m = -INFINITY, l = 0.f;
  uint32_t phase = 0;
  // staging roles: K row kr = t >> 1, dims d0 .. d0 + 15; Vᵀ row = dim `lane`, keys w·16 .. + 15
  const int kr = t >> 1, d0 = (t & 1) * 16, vk0 = warp * 16;
  float4 kx[4];
  float vx[16];
  auto load_block = [&](int kb) {
    const long key = long(kb) + kr;
    const bool ok = key < kend;
#pragma unroll
    for (int c = 0; c < 4; ++c)
      kx[c] = ok ? __ldg(reinterpret_cast<const float4 *>(a.K + key * D + hc + d0) + c)
                 : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int c = 0; c < 16; ++c) {
      const long kv = long(kb) + vk0 + c;
      vx[c] = kv < kend ? __ldg(a.V + kv * D + hc + lane) : 0.f;
    }
  };
  if (kbeg < kend) load_block(kbeg);
  for (int kb = kbeg; kb < kend; kb += KB) {
    {   // ---- stage the prefetched block: K (SW128 K-major, rows = keys), Vᵀ (rows = dims)
      uint32_t h[8], lw[8];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        if constexpr (SPLIT) {
          split_h2(kx[c].x, kx[c].y, h[2 * c], lw[2 * c]);
          split_h2(kx[c].z, kx[c].w, h[2 * c + 1], lw[2 * c + 1]);
        } else {
          h[2 * c] = pack_h2(kx[c].x, kx[c].y);
          h[2 * c + 1] = pack_h2(kx[c].z, kx[c].w);
        }
      }
      *reinterpret_cast<uint4 *>(Kh + tc::sw128_offset_f16(kr, d0, KB)) = make_uint4(h[0], h[1], h[2], h[3]);
      *reinterpret_cast<uint4 *>(Kh + tc::sw128_offset_f16(kr, d0 + 8, KB)) = make_uint4(h[4], h[5], h[6], h[7]);
      if constexpr (SPLIT) {
        *reinterpret_cast<uint4 *>(Kl + tc::sw128_offset_f16(kr, d0, KB)) = make_uint4(lw[0], lw[1], lw[2], lw[3]);
        *reinterpret_cast<uint4 *>(Kl + tc::sw128_offset_f16(kr, d0 + 8, KB)) = make_uint4(lw[4], lw[5], lw[6], lw[7]);
      }
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        if constexpr (SPLIT) split_h2(vx[2 * c], vx[2 * c + 1], h[c], lw[c]);
        else h[c] = pack_h2(vx[2 * c], vx[2 * c + 1]);
      }
      *reinterpret_cast<uint4 *>(Vh + tc::sw128_offset_f16(lane, vk0, 32)) = make_uint4(h[0], h[1], h[2], h[3]);
      *reinterpret_cast<uint4 *>(Vh + tc::sw128_offset_f16(lane, vk0 + 8, 32)) = make_uint4(h[4], h[5], h[6], h[7]);
      if constexpr (SPLIT) {
        *reinterpret_cast<uint4 *>(Vl + tc::sw128_offset_f16(lane, vk0, 32)) = make_uint4(lw[0], lw[1], lw[2], lw[3]);
        *reinterpret_cast<uint4 *>(Vl + tc::sw128_offset_f16(lane, vk0 + 8, 32)) = make_uint4(lw[4], lw[5], lw[6], lw[7]);
      }
    }
    fence_proxy_async_smem();
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    if (t == 0) {     // ---- S = Q Kᵀ (N = 64, K = 32: two k16 steps)
#pragma unroll
      for (int kk = 0; kk < 2; ++kk) {
        const uint64_t bh = tc::sdesc_sw128(kh_a + kk * 32), bl = tc::sdesc_sw128(kl_a + kk * 32);
        if constexpr (SPLIT) {
          tc::mma_f16_ts(tmem + SC, tmem + QL + kk * 8, bh, id_s, kk > 0 ? 1u : 0u);
          tc::mma_f16_ts(tmem + SC, tmem + QH + kk * 8, bl, id_s, 1u);
          tc::mma_f16_ts(tmem + SC, tmem + QH + kk * 8, bh, id_s, 1u);
        } else {
          (void)bl;
          tc::mma_f16_ts(tmem + SC, tmem + QH + kk * 8, bh, id_s, kk > 0 ? 1u : 0u);
        }
      }
      tc::mma_commit(bar);
    }
    if (kb + KB < kend) load_block(kb + KB);        // next block's K / V in flight meanwhile
    mbar_spin(bar, phase);
    phase ^= 1;
    tc::fence_after_sync();
    {   // ---- online softmax on this thread's row (P overwrites S in TMEM)
      uint32_t s0[32], s1[32];
      tc::tmem_ld32(lane_base + SC, s0);
      tc::tmem_ld32(lane_base + SC + 32, s1);
      tc::tmem_ld_wait();
      float bm = -INFINITY;
      if (!__all_sync(0xffffffffu, kb >= lo && kb + KB <= hi)) {   // mask keys outside the row's graph
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          if (!(kb + j >= lo && kb + j < hi)) s0[j] = __float_as_uint(-INFINITY);
          if (!(kb + 32 + j >= lo && kb + 32 + j < hi)) s1[j] = __float_as_uint(-INFINITY);
        }
      }
#pragma unroll
      for (int j = 0; j < 32; ++j) bm = fmaxf(bm, fmaxf(__uint_as_float(s0[j]), __uint_as_float(s1[j])));
      const float mn = fmaxf(m, bm);
      const float ref = mn == -INFINITY ? 0.f : mn;
      const float f = ex2f(m - ref);
      m = mn;
      float sum = 0.f;
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {         // P in two 16-column halves (fewer live registers)
        uint32_t ph[16], pl[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const uint32_t *src = hf == 0 ? s0 : s1;
          const float p0 = ex2f(__uint_as_float(src[2 * j]) - ref);
          const float p1 = ex2f(__uint_as_float(src[2 * j + 1]) - ref);
          sum += p0 + p1;
          if constexpr (SPLIT) split_h2(p0, p1, ph[j], pl[j]);
          else ph[j] = pack_h2(p0, p1);
        }
        tc::tmem_st16(lane_base + PH + 16 * hf, ph);
        if constexpr (SPLIT) tc::tmem_st16(lane_base + PL + 16 * hf, pl);
      }
      l = l * f + sum;
      if (__any_sync(0xffffffffu, f != 1.f)) {     // rescale the O row (warp-collective)
        uint32_t o[32];
        tc::tmem_ld32(lane_base + OC, o);
        tc::tmem_ld_wait();
#pragma unroll
        for (int c = 0; c < 32; ++c) o[c] = __float_as_uint(__uint_as_float(o[c]) * f);
        tc::tmem_st32(lane_base + OC, o);
      }
      tc::tmem_st_wait();
    }
    tc::fence_before_sync();
    __syncthreads();
    tc::fence_after_sync();
    if (t == 0) {     // ---- O += P V (N = 32, K = 64 keys: four k16 steps)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const uint64_t bh = tc::sdesc_sw128(vh_a + kk * 32), bl = tc::sdesc_sw128(vl_a + kk * 32);
        if constexpr (SPLIT) {
          tc::mma_f16_ts(tmem + OC, tmem + PL + kk * 8, bh, id_o, 1u);
          tc::mma_f16_ts(tmem + OC, tmem + PH + kk * 8, bl, id_o, 1u);
        } else {
          (void)bl;
        }
        tc::mma_f16_ts(tmem + OC, tmem + PH + kk * 8, bh, id_o, 1u);
      }
      tc::mma_commit(bar);
    }
    mbar_spin(bar, phase);
    phase ^= 1;
    tc::fence_after_sync();
  }
  {   // ---- O / l -> global
    uint32_t o[32];
    tc::tmem_ld32(lane_base + OC, o);
    tc::tmem_ld_wait();
    const float il = l > 0.f ? 1.f / l : 0.f;
    if (live) {
#pragma unroll
      for (int c = 0; c < 32; c += 4)
        *reinterpret_cast<float4 *>(a.O + r * D + hc + c) =
            make_float4(__uint_as_float(o[c]) * il, __uint_as_float(o[c + 1]) * il,
                        __uint_as_float(o[c + 2]) * il, __uint_as_float(o[c + 3]) * il);
    }
  }
  tc::fence_before_sync();
  __syncthreads();
  if (warp == 0) tc::tmem_dealloc<TCOLS>(tmem);
}

template <int D>
int ln_launch(const occu_ctx *ctx, const float *X, int N, const float *g, const float *b, float *Y,
              cudaStream_t st) {
  OCCU_PROF_BEGIN(ctx, "gph_ln", st);
  gph_ln_kernel<D><<<(N + 7) / 8, 256, 0, st>>>(X, N, g, b, Y);
  OCCU_PROF_END(ctx);
  return 1;
}

}  // namespace

int launch_graphormer_layer(const occu_ctx *ctx, const DevCsr &csr, int j, const float *h_in,
                            float *h_out, float *X, float *QKV, float *O, cudaStream_t st,
                            const GphSave *sv) {
  const occu_config &cf = ctx->cfg;
  const GphOff &G = ctx->layout.G[j];
  const float *P = ctx->params.as<float>();
  const int D = cf.d, N = csr.N, slot = cf.L + 1 + j;
  if (N <= 0) return 0;
  const size_t ND = size_t(N) * D;
  float *Qb = QKV, *Kb = QKV + ND, *Vb = QKV + 2 * ND;
  float *X2 = X, *Hb = Kb, *T = Qb;        // inference: scratch reused stage by stage
  if (sv) {                                 // training: every intermediate kept (backward)
    X = sv->X1; Qb = sv->Q; Kb = sv->K; Vb = sv->V; O = sv->O;
    Hb = sv->Hb; X2 = sv->X2; T = sv->T;
  }
  int n = 0, r;
  auto ln = [&](const float *x, size_t g, size_t b, float *y) {
    return D == 64 ? ln_launch<64>(ctx, x, N, P + g, P + b, y, st)
                   : ln_launch<128>(ctx, x, N, P + g, P + b, y, st);
  };
  // h̄ = MHA(LN(h)) + h
  n += ln(h_in, G.ln1_g, G.ln1_b, X);
  if ((r = launch_bias_tc(ctx, X, D, N, 0, slot, P + G.bq, false, Qb, "gph_qkv_tc", st)) < 0) return r;
  n += r;
  if ((r = launch_bias_tc(ctx, X, D, N, 1, slot, P + G.bk, false, Kb, "gph_qkv_tc", st)) < 0) return r;
  n += r;
  if ((r = launch_bias_tc(ctx, X, D, N, 2, slot, P + G.bv, false, Vb, "gph_qkv_tc", st)) < 0) return r;
  n += r;
  AttnArgs a;
  a.Q = Qb; a.K = Kb; a.V = Vb; a.node_off = csr.node_off; a.node_graph = csr.node_graph;
  a.O = O; a.N = N; a.D = D;
  const int dh = D / cf.heads;
  a.qscale = L2E / sqrtf(float(dh));
  const dim3 grid((N + QT - 1) / QT, cf.heads);
  OCCU_PROF_BEGIN(ctx, "gph_attn", st);
  auto go = [&](auto kern, int DH) {
    const size_t smem = size_t(4) * KT * (DH + 4) * sizeof(float);
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    kern<<<grid, AW * 32, smem, st>>>(a);
  };
  static const bool tf32 = [] {
    const char *e = getenv("OCCU_GPH_TF32");
    return e && atoi(e) != 0;
  }();
  auto goh = [&](auto kern, size_t smem) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    kern<<<grid, AW * 32, smem, st>>>(a);
  };
  static const bool use_tc = [] {
    const char *e = getenv("OCCU_GPH_TC");
    return !e || atoi(e) != 0;
  }();
  if (use_tc && dh == 32 && !tf32) {    // tcgen05 path (d_h = 32)
    const dim3 g2((N + 127) / 128, cf.heads);
    if (cf.prec == OCCU_BF16) {         // R42: one fp16 product per step
      cudaFuncSetAttribute(gph_attn_tc_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(gtc::SMEM));
      gph_attn_tc_kernel<false><<<g2, 128, gtc::SMEM, st>>>(a);
    } else {
      cudaFuncSetAttribute(gph_attn_tc_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(gtc::SMEM));
      gph_attn_tc_kernel<true><<<g2, 128, gtc::SMEM, st>>>(a);
    }
  } else if (tf32) {       // A/B: the TF32-split variant
    switch (dh) {
      case 16: go(gph_attn_kernel<16>, 16); break;
      case 32: go(gph_attn_kernel<32>, 32); break;
      case 64: go(gph_attn_kernel<64>, 64); break;
      default: return -int(cudaErrorInvalidValue);
    }
  } else {
    switch (dh) {
      case 16: goh(gph_attn_f16_kernel<16>, F16Smem<16>::bytes); break;
      case 32: goh(gph_attn_f16_kernel<32>, F16Smem<32>::bytes); break;
      case 64: goh(gph_attn_f16_kernel<64>, F16Smem<64>::bytes); break;
      default: return -int(cudaErrorInvalidValue);
    }
  }
  OCCU_PROF_END(ctx);
  ++n;
  // h̄ (inference: K is dead after the attention, h̄ lives there)
  if ((r = launch_bias_add_tc(ctx, O, D, N, 3, slot, P + G.bo, h_in, Hb, "gph_out_tc", st)) < 0) return r;
  n += r;
  // h' = FFN(LN(h̄)) + h̄
  n += ln(Hb, G.ln2_g, G.ln2_b, X2);
  // FFN hidden rows (inference: in Q's place)
  if ((r = launch_bias_tc(ctx, X2, D, N, 4, slot, P + G.F.b1, true, T, "gph_ffn_tc", st)) < 0) return r;
  n += r;
  if ((r = launch_bias_add_tc(ctx, T, D, N, 5, slot, P + G.F.b2, Hb, h_out, "gph_ffn_tc", st)) < 0) return r;
  n += r;
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? n : -int(e);
}

}  // namespace occu
