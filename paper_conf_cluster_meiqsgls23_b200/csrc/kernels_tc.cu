// Tensor-core (tcgen05) forward kernels for the FP32 path, sm_100a.
//
// Every dense contraction of an ANEE layer (P141 W_u, P145 W_e, P149 W_m) runs
// on the 5th-generation tensor cores as a 3xTF32 product (x = x_hi + x_lo with
// x_hi = tf32(x): x·w ≈ x_hi·w_hi + x_hi·w_lo + x_lo·w_hi, FP32 accumulation in
// TMEM), which keeps FP32-level accuracy (~1e-6 relative).
//
// Structure of one CTA (128 threads = 4 warps, persistent over 128-row tiles):
//   * the layer's weight matrix W [D][K] is split once per CTA into hi / lo
//     tf32 images in shared memory, K-major 128-byte-swizzle layout (the UMMA B
//     operand);
//   * a tile of 128 rows (nodes or in-CSR-ordered edges) is staged with
//     coalesced 16-byte loads into padded shared memory, each thread takes its
//     row, splits it and writes hi / lo into TMEM with tcgen05.st (the UMMA A
//     operand, ".ts" form: A from tensor memory);
//   * one elected thread issues 3 x K/8 tcgen05.mma (M=128, N=D, K=8) into a
//     TMEM accumulator and commits to an mbarrier;
//   * the epilogue reads its accumulator row with tcgen05.ld (thread = row):
//       node_tc      : h̄ = LReLU(.), p = h̄·a_s, q = h̄·a_d            (a2)
//       edge_tc      : e' = σ((p[s] + q[t]) · .)                      (a3)
//       gate_agg_tc  : g = softmax_c(.), m = g ⊙ h̄[s], then a column-
//                      ordered segmented sum over the destination-sorted
//                      tile -> h = LReLU(Σ m) (a4, a5, a6); segments that
//                      cross a tile boundary leave fixed-slot partials that
//                      fixup_kernel combines in tile order (no atomics).
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>

#include "occu_internal.h"
#include "tc_common.cuh"

namespace occu {
namespace {

constexpr int TM = 128;          // rows per tile (UMMA M)
constexpr int NTH = 128;         // threads per CTA
constexpr uint32_t A_HI_COL = 0, A_LO_COL = 128, ACC_COL = 256, TMEM_COLS = 512;

__device__ __forceinline__ float lrelu(float x, float s) { return x > 0.f ? x : s * x; }

struct SmemLayout {
  uint32_t w_hi, w_lo, stage, misc, extra, total;
};
// Offsets (bytes from the 1024-aligned base): W images, staging tile, misc
// (mbarrier, TMEM slot, per-tile indices), extra (plain fp32 weights, SIMT z).
__host__ __device__ inline SmemLayout smem_layout(int D, int Kpad, int S, int extra_bytes = 0) {
  SmemLayout L;
  const uint32_t img = uint32_t(Kpad) * D * 4;
  L.w_hi = 0;
  L.w_lo = img;
  L.stage = 2 * img;
  L.misc = L.stage + uint32_t(TM) * S * 4;
  L.extra = L.misc + 1024;
  L.total = L.extra + uint32_t(extra_bytes);
  return L;
}

// W [D][K] (row n = output channel, K-major) -> hi / lo SW128 images in smem.
__device__ void load_weight_images(uint8_t *base, const SmemLayout &L,
                                   const float *__restrict__ W, int D, int K, int Kpad) {
  uint32_t *hi = reinterpret_cast<uint32_t *>(base + L.w_hi);
  uint32_t *lo = reinterpret_cast<uint32_t *>(base + L.w_lo);
  for (int idx = threadIdx.x; idx < D * Kpad; idx += NTH) {
    const int n = idx / Kpad, k = idx % Kpad;
    const float v = k < K ? __ldg(W + long(n) * K + k) : 0.f;
    uint32_t h, l;
    tc::split_tf32(v, h, l);
    const uint32_t off = tc::sw128_offset_f32(n, k, D) >> 2;
    hi[off] = h;
    lo[off] = l;
  }
}

// Coalesced copy of rows [row0, row0+nrows) of A [*, K] into stage (stride S floats).
__device__ __forceinline__ void stage_rows(float *stage, int S, const float *__restrict__ A,
                                           long row0, int nrows, int K) {
  const int kq = K >> 2;
  const int total = TM * kq;
  const float4 *src = reinterpret_cast<const float4 *>(A + row0 * K);
#pragma unroll 4
  for (int f = threadIdx.x; f < total; f += NTH) {
    const int r = f / kq, c = f - r * kq;
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (r < nrows) v = __ldg(src + f);
    *reinterpret_cast<float4 *>(stage + r * S + c * 4) = v;
  }
}

// Thread's own staged row -> hi/lo tf32 into TMEM A columns (Kpad columns, zero padded).
__device__ __forceinline__ void row_to_tmem_a(const float *row, int K, int Kpad, uint32_t tmem_lane) {
  for (int c0 = 0; c0 < Kpad; c0 += 32) {
    uint32_t hi[32], lo[32];
#pragma unroll
    for (int j = 0; j < 32; j += 4) {
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (c0 + j < K) v = *reinterpret_cast<const float4 *>(row + c0 + j);
      tc::split_tf32(v.x, hi[j], lo[j]);
      tc::split_tf32(v.y, hi[j + 1], lo[j + 1]);
      tc::split_tf32(v.z, hi[j + 2], lo[j + 2]);
      tc::split_tf32(v.w, hi[j + 3], lo[j + 3]);
    }
    tc::tmem_st32(tmem_lane + A_HI_COL + c0, hi);
    tc::tmem_st32(tmem_lane + A_LO_COL + c0, lo);
  }
  tc::tmem_st_wait();
}

// 3xTF32 MMA chain: ACC = A_hi·W_hi + A_hi·W_lo + A_lo·W_hi over Kpad.
__device__ __forceinline__ void issue_mma_3xtf32(uint32_t tmem, uint32_t whi_addr, uint32_t wlo_addr,
                                                 int D, int Kpad, uint64_t *bar) {
  const uint32_t idsc = tc::idesc(128, uint32_t(D), tc::FMT_TF32);
  for (int kk = 0; kk < Kpad / 8; ++kk) {
    const uint32_t boff = uint32_t(kk >> 2) * uint32_t(D) * 128u + uint32_t(kk & 3) * 32u;
    const uint64_t bh = tc::sdesc_sw128(whi_addr + boff);
    const uint64_t bl = tc::sdesc_sw128(wlo_addr + boff);
    const uint32_t ah = tmem + A_HI_COL + kk * 8, al = tmem + A_LO_COL + kk * 8;
    tc::mma_tf32_ts(tmem + ACC_COL, ah, bh, idsc, kk > 0 ? 1u : 0u);
    tc::mma_tf32_ts(tmem + ACC_COL, ah, bl, idsc, 1u);
    tc::mma_tf32_ts(tmem + ACC_COL, al, bh, idsc, 1u);
  }
  tc::mma_commit(bar);
}

// Write row r (D floats in v) into the staging tile, then the block copies the
// staged tile to dst rows [row0, row0+nrows) coalesced.
__device__ __forceinline__ void flush_stage(const float *stage, int S, float *__restrict__ dst,
                                            long row0, int nrows, int D) {
  const int dq = D >> 2;
  float4 *out = reinterpret_cast<float4 *>(dst + row0 * D);
  for (int f = threadIdx.x; f < nrows * dq; f += NTH) {
    const int r = f / dq, c = f - r * dq;
    out[f] = *reinterpret_cast<const float4 *>(stage + r * S + c * 4);
  }
}

struct TileCtx {
  uint8_t *base;
  SmemLayout L;
  uint64_t *bar;
  uint32_t *tmem_slot;
};

__device__ __forceinline__ TileCtx setup(uint8_t *raw, const SmemLayout &L) {
  TileCtx t;
  const uint32_t a = tc::smem_u32(raw);
  t.base = raw + ((1024 - (a & 1023)) & 1023);
  t.L = L;
  t.bar = reinterpret_cast<uint64_t *>(t.base + L.misc);
  t.tmem_slot = reinterpret_cast<uint32_t *>(t.base + L.misc + 64);
  if (threadIdx.x == 0) {
    tc::mbar_init(t.bar, 1);
    tc::fence_mbar_init();
  }
  if (threadIdx.x < 32) tc::tmem_alloc<TMEM_COLS>(t.tmem_slot);
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  return t;
}

__device__ __forceinline__ void teardown(const TileCtx &t) {
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  if (threadIdx.x < 32) tc::tmem_dealloc<TMEM_COLS>(*t.tmem_slot);
}

// Stage A rows, move them to TMEM, run the MMA chain, wait for the accumulator.
__device__ __forceinline__ void tile_gemm(const TileCtx &t, float *stage, int S,
                                          const float *__restrict__ A, long row0, int nrows,
                                          int K, int Kpad, int D, uint32_t &phase) {
  const uint32_t tmem = *t.tmem_slot;
  const int warp = threadIdx.x >> 5;
  const uint32_t lane_addr = tmem + (uint32_t(warp * 32) << 16);
  stage_rows(stage, S, A, row0, nrows, K);
  __syncthreads();
  row_to_tmem_a(stage + threadIdx.x * S, K, Kpad, lane_addr);
  tc::fence_before_sync();
  __syncthreads();
  if (threadIdx.x == 0) {
    tc::fence_after_sync();
    issue_mma_3xtf32(tmem, tc::smem_u32(t.base + t.L.w_hi), tc::smem_u32(t.base + t.L.w_lo), D,
                     Kpad, t.bar);
  }
  tc::mbar_wait(t.bar, phase);
  phase ^= 1u;
  tc::fence_after_sync();
}

// ---------------------------------------------------------------------------
// a2: h̄ = LReLU(h W_uᵀ), p = h̄·a_s, q = h̄·a_d
// ---------------------------------------------------------------------------
template <int D>
__global__ void __launch_bounds__(NTH, 1)
node_tc_kernel(const float *__restrict__ A, int K, int Kpad, const float *__restrict__ W,
               const float *__restrict__ a_s, const float *__restrict__ a_d, int N, float slope,
               float *__restrict__ hbar, float *__restrict__ p, float *__restrict__ q) {
  extern __shared__ uint8_t smem_raw[];
  const int S = (K > D ? K : D) + 4;
  const SmemLayout L = smem_layout(D, Kpad, S);
  TileCtx t = setup(smem_raw, L);
  load_weight_images(t.base, L, W, D, K, Kpad);
  __syncthreads();
  float *stage = reinterpret_cast<float *>(t.base + L.stage);
  const uint32_t tmem = *t.tmem_slot;
  const uint32_t lane_addr = tmem + (uint32_t((threadIdx.x >> 5) * 32) << 16);
  uint32_t phase = 0;
  const int tiles = (N + TM - 1) / TM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long r0 = long(tile) * TM;
    const int nrows = min(TM, int(N - r0));
    tile_gemm(t, stage, S, A, r0, nrows, K, Kpad, D, phase);
    // epilogue: thread = row
    float pp = 0.f, qq = 0.f;
    float *myrow = stage + threadIdx.x * S;
#pragma unroll
    for (int c0 = 0; c0 < D; c0 += 32) {
      uint32_t r[32];
      tc::tmem_ld32(lane_addr + ACC_COL + c0, r);
      tc::tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 32; j += 4) {
        float4 v;
        v.x = lrelu(__uint_as_float(r[j]), slope);
        v.y = lrelu(__uint_as_float(r[j + 1]), slope);
        v.z = lrelu(__uint_as_float(r[j + 2]), slope);
        v.w = lrelu(__uint_as_float(r[j + 3]), slope);
        const float4 as4 = __ldg(reinterpret_cast<const float4 *>(a_s + c0 + j));
        const float4 ad4 = __ldg(reinterpret_cast<const float4 *>(a_d + c0 + j));
        pp = fmaf(v.x, as4.x, pp); pp = fmaf(v.y, as4.y, pp);
        pp = fmaf(v.z, as4.z, pp); pp = fmaf(v.w, as4.w, pp);
        qq = fmaf(v.x, ad4.x, qq); qq = fmaf(v.y, ad4.y, qq);
        qq = fmaf(v.z, ad4.z, qq); qq = fmaf(v.w, ad4.w, qq);
        *reinterpret_cast<float4 *>(myrow + c0 + j) = v;
      }
    }
    if (threadIdx.x < nrows) {
      p[r0 + threadIdx.x] = pp;
      q[r0 + threadIdx.x] = qq;
    }
    tc::fence_before_sync();
    __syncthreads();
    flush_stage(stage, S, hbar, r0, nrows, D);
    __syncthreads();
  }
  teardown(t);
}

// ---------------------------------------------------------------------------
// a3: e' = σ((p[s] + q[t]) · W_e e).  Layer 1 (Ke = F_e small): z on CUDA cores.
// ---------------------------------------------------------------------------
template <int D, bool TCZ>
__global__ void __launch_bounds__(NTH, 1)
edge_tc_kernel(const float *__restrict__ e_in, int Ke, int Kpad, const float *__restrict__ W_e,
               const float *__restrict__ p, const float *__restrict__ q,
               const int32_t *__restrict__ in_src, const int32_t *__restrict__ in_dst, int E,
               float *__restrict__ e_out) {
  extern __shared__ uint8_t smem_raw[];
  const int S = (Ke > D ? Ke : D) + 4;
  const SmemLayout L = smem_layout(D, TCZ ? Kpad : 0, S, TCZ ? 0 : D * Ke * 4);
  TileCtx t = setup(smem_raw, L);
  float *wsimt = reinterpret_cast<float *>(t.base + L.extra);  // [D][Ke] fp32 (SIMT z)
  if (TCZ) {
    load_weight_images(t.base, L, W_e, D, Ke, Kpad);
  }
  float *stage = reinterpret_cast<float *>(t.base + L.stage);
  __syncthreads();
  if (!TCZ) {
    for (int i = threadIdx.x; i < D * Ke; i += NTH) wsimt[i] = W_e[i];
    __syncthreads();
  }
  const uint32_t tmem = *t.tmem_slot;
  const uint32_t lane_addr = tmem + (uint32_t((threadIdx.x >> 5) * 32) << 16);
  uint32_t phase = 0;
  const int tiles = (E + TM - 1) / TM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long k0 = long(tile) * TM;
    const int nrows = min(TM, int(E - k0));
    const int r = threadIdx.x;
    float alpha = 0.f;
    if (r < nrows) alpha = p[in_src[k0 + r]] + q[in_dst[k0 + r]];       // R1
    float *myrow = stage + r * S;
    if (TCZ) {
      tile_gemm(t, stage, S, e_in, k0, nrows, Ke, Kpad, D, phase);
#pragma unroll
      for (int c0 = 0; c0 < D; c0 += 32) {
        uint32_t v[32];
        tc::tmem_ld32(lane_addr + ACC_COL + c0, v);
        tc::tmem_ld_wait();
#pragma unroll
        for (int j = 0; j < 32; j += 4) {
          float4 o;
          o.x = 1.f / (1.f + expf(-(alpha * __uint_as_float(v[j]))));
          o.y = 1.f / (1.f + expf(-(alpha * __uint_as_float(v[j + 1]))));
          o.z = 1.f / (1.f + expf(-(alpha * __uint_as_float(v[j + 2]))));
          o.w = 1.f / (1.f + expf(-(alpha * __uint_as_float(v[j + 3]))));
          *reinterpret_cast<float4 *>(myrow + c0 + j) = o;
        }
      }
      tc::fence_before_sync();
    } else {
      // z[c] = Σ_k W_e[c][k] e[k], k < Ke (Ke <= 16), fp32 FMA in ascending k
      float e[16];
#pragma unroll
      for (int k = 0; k < 16; ++k) e[k] = 0.f;
      if (r < nrows)
        for (int k = 0; k < Ke; ++k) e[k] = __ldg(e_in + (k0 + r) * Ke + k);
      __syncthreads();   // previous tile's flush finished with the stage
      for (int c = 0; c < D; c += 4) {
        float o[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const float *w = wsimt + (c + u) * Ke;
          float z = 0.f;
          for (int k = 0; k < Ke; ++k) z = fmaf(w[k], e[k], z);
          o[u] = 1.f / (1.f + expf(-(alpha * z)));
        }
        *reinterpret_cast<float4 *>(myrow + c) = make_float4(o[0], o[1], o[2], o[3]);
      }
    }
    __syncthreads();
    flush_stage(stage, S, e_out, k0, nrows, D);
    __syncthreads();
  }
  teardown(t);
}

// ---------------------------------------------------------------------------
// a4 + a5 + a6: g = softmax_c(W_m e'), m = g ⊙ h̄[s], h[t] = LReLU(Σ_seg m)
// ---------------------------------------------------------------------------
template <int D>
__global__ void __launch_bounds__(NTH, 1)
gate_agg_tc_kernel(const float *__restrict__ e, const float *__restrict__ W_m,
                   const float *__restrict__ hbar, const int32_t *__restrict__ in_src,
                   const int32_t *__restrict__ in_dst, const int32_t *__restrict__ in_ptr, int E,
                   int mean, float slope, float *__restrict__ h_out, float *__restrict__ partial) {
  extern __shared__ uint8_t smem_raw[];
  const int S = D + 4;
  const SmemLayout L = smem_layout(D, D, S);
  TileCtx t = setup(smem_raw, L);
  load_weight_images(t.base, L, W_m, D, D, D);
  float *stage = reinterpret_cast<float *>(t.base + L.stage);
  int *dst_s = reinterpret_cast<int *>(t.base + L.misc + 128);     // [TM]
  __syncthreads();
  const uint32_t tmem = *t.tmem_slot;
  const uint32_t lane_addr = tmem + (uint32_t((threadIdx.x >> 5) * 32) << 16);
  uint32_t phase = 0;
  const int tiles = (E + TM - 1) / TM;
  for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const long k0 = long(tile) * TM;
    const int nrows = min(TM, int(E - k0));
    const int r = threadIdx.x;
    int src = 0;
    if (r < nrows) {
      src = in_src[k0 + r];
      dst_s[r] = in_dst[k0 + r];
    } else {
      dst_s[r] = -1;
    }
    tile_gemm(t, stage, S, e, k0, nrows, D, D, D, phase);
    // softmax over the D channels of this edge's row (thread-local)
    float mx = -INFINITY;
#pragma unroll
    for (int c0 = 0; c0 < D; c0 += 32) {
      uint32_t v[32];
      tc::tmem_ld32(lane_addr + ACC_COL + c0, v);
      tc::tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 32; ++j) mx = fmaxf(mx, __uint_as_float(v[j]));
    }
    float *myrow = stage + r * S;
    float sum = 0.f;
#pragma unroll
    for (int c0 = 0; c0 < D; c0 += 32) {
      uint32_t v[32];
      tc::tmem_ld32(lane_addr + ACC_COL + c0, v);
      tc::tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 32; j += 4) {
        float4 x;
        x.x = expf(__uint_as_float(v[j]) - mx);
        x.y = expf(__uint_as_float(v[j + 1]) - mx);
        x.z = expf(__uint_as_float(v[j + 2]) - mx);
        x.w = expf(__uint_as_float(v[j + 3]) - mx);
        sum += x.x; sum += x.y; sum += x.z; sum += x.w;
        *reinterpret_cast<float4 *>(myrow + c0 + j) = x;
      }
    }
    const float *hr = hbar + long(src) * D;
    const bool live = r < nrows;
#pragma unroll 4
    for (int c = 0; c < D; c += 4) {
      const float4 x = *reinterpret_cast<const float4 *>(myrow + c);
      float4 hb = make_float4(0.f, 0.f, 0.f, 0.f);
      if (live) hb = __ldg(reinterpret_cast<const float4 *>(hr + c));
      float4 m;
      m.x = (x.x / sum) * hb.x;
      m.y = (x.y / sum) * hb.y;
      m.z = (x.z / sum) * hb.z;
      m.w = (x.w / sum) * hb.w;
      *reinterpret_cast<float4 *>(myrow + c) = m;
    }
    tc::fence_before_sync();
    __syncthreads();
    // column-ordered segmented sum: thread c owns channel c
    for (int c = threadIdx.x; c < D; c += NTH) {
      int tprev = dst_s[0];
      float acc = 0.f;
      for (int k = 0; k <= nrows; ++k) {
        const int tcur = k < nrows ? dst_s[k] : -2;
        if (tcur != tprev) {
          const int beg = in_ptr[tprev], end = in_ptr[tprev + 1];
          const bool before = beg < k0, after = end > k0 + nrows;
          if (!before && !after) {
            float a = acc;
            if (mean) a = a / float(end - beg);
            h_out[long(tprev) * D + c] = lrelu(a, slope);
          } else {
            partial[(long(tile) * 2 + (before ? 0 : 1)) * D + c] = acc;
          }
          acc = 0.f;
          tprev = tcur;
        }
        if (k < nrows) acc += stage[k * S + c];
      }
    }
    __syncthreads();
  }
  teardown(t);
}

// Nodes whose in-edge segment spans tiles: combine fixed-slot partials in tile
// order; nodes without in-edges: h = LReLU(0) = 0 (R8).
__global__ void fixup_kernel(const int32_t *__restrict__ in_ptr, int N, int D,
                             const float *__restrict__ partial, int mean, float slope,
                             float *__restrict__ h_out) {
  const long total = long(N) * D;
  for (long i = blockIdx.x * long(blockDim.x) + threadIdx.x; i < total;
       i += long(gridDim.x) * blockDim.x) {
    const int t = int(i / D), c = int(i % D);
    const int beg = in_ptr[t], end = in_ptr[t + 1];
    if (beg == end) {
      h_out[i] = 0.f;
      continue;
    }
    const int tb = beg / TM, te = (end - 1) / TM;
    if (tb == te) continue;
    float s = partial[(long(tb) * 2 + 1) * D + c];
    for (int T = tb + 1; T <= te; ++T) s += partial[(long(T) * 2 + 0) * D + c];
    if (mean) s = s / float(end - beg);
    h_out[i] = lrelu(s, slope);
  }
}

inline int grid_tiles(long rows, int sms) {
  long tiles = (rows + TM - 1) / TM;
  return int(std::max<long>(1, std::min<long>(tiles, sms)));
}

template <class Kern> void set_smem(Kern k, size_t bytes) {
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes));
}

}  // namespace

#define TC_CHECK()                                  \
  do {                                              \
    cudaError_t e_ = cudaGetLastError();            \
    if (e_ != cudaSuccess) return -int(e_);         \
  } while (0)

bool tc_supported(const occu_config &c) {
  return (c.d == 64 || c.d == 128) && c.F_n <= 128;
}

size_t tc_partial_floats(int E, int D) { return size_t((E + TM - 1) / TM + 1) * 2 * D; }

template <int D>
static int tc_forward_layer_impl(const occu_ctx *ctx, const DevCsr &csr, const FwdLayerArgs &a,
                                 float *partial, cudaStream_t st) {
  const int sms = ctx->num_sms;
  const float slope = ctx->cfg.slope;
  const int mean = ctx->cfg.aggr == OCCU_AGGR_MEAN;
  int n = 0;
  if (csr.N > 0) {
    const int Kpad = (a.K + 31) / 32 * 32;
    const int S = std::max(a.K, D) + 4;
    const size_t smem = smem_layout(D, Kpad, S).total + 1024;
    set_smem(node_tc_kernel<D>, smem);
    OCCU_PROF_BEGIN(ctx, "node_tc", st);
    node_tc_kernel<D><<<grid_tiles(csr.N, sms), NTH, smem, st>>>(
        a.h_in, a.K, Kpad, a.W_u, a.a_s, a.a_d, csr.N, slope, a.hbar, a.p, a.q);
    OCCU_PROF_END(ctx);
    TC_CHECK();
    ++n;
  }
  if (csr.E > 0) {
    const bool tcz = a.Ke > 16;
    const int Kpad = (a.Ke + 31) / 32 * 32;
    const int S = std::max(a.Ke, D) + 4;
    OCCU_PROF_BEGIN(ctx, "edge_tc", st);
    if (tcz) {
      const size_t smem = smem_layout(D, Kpad, S).total + 1024;
      set_smem(edge_tc_kernel<D, true>, smem);
      edge_tc_kernel<D, true><<<grid_tiles(csr.E, sms), NTH, smem, st>>>(
          a.e_in, a.Ke, Kpad, a.W_e, a.p, a.q, csr.in_src, csr.in_dst, csr.E, a.e_out);
    } else {
      const size_t smem = smem_layout(D, 0, S, D * a.Ke * 4).total + 1024;
      set_smem(edge_tc_kernel<D, false>, smem);
      edge_tc_kernel<D, false><<<grid_tiles(csr.E, sms), NTH, smem, st>>>(
          a.e_in, a.Ke, 0, a.W_e, a.p, a.q, csr.in_src, csr.in_dst, csr.E, a.e_out);
    }
    OCCU_PROF_END(ctx);
    TC_CHECK();
    ++n;
    const size_t smem = smem_layout(D, D, D + 4).total + 1024;
    set_smem(gate_agg_tc_kernel<D>, smem);
    OCCU_PROF_BEGIN(ctx, "gate_agg_tc", st);
    gate_agg_tc_kernel<D><<<grid_tiles(csr.E, sms), NTH, smem, st>>>(
        a.e_out, a.W_m, a.hbar, csr.in_src, csr.in_dst, csr.in_ptr, csr.E, mean, slope, a.h_out,
        partial);
    OCCU_PROF_END(ctx);
    TC_CHECK();
    ++n;
  }
  if (csr.N > 0) {
    const long total = long(csr.N) * D;
    const int grid = int(std::min<long>((total + 255) / 256, 16L * sms));
    OCCU_PROF_BEGIN(ctx, "fixup", st);
    fixup_kernel<<<grid, 256, 0, st>>>(csr.in_ptr, csr.N, D, partial, mean, slope, a.h_out);
    OCCU_PROF_END(ctx);
    TC_CHECK();
    ++n;
  }
  return n;
}

int launch_forward_layer_tc(const occu_ctx *ctx, const DevCsr &csr, const FwdLayerArgs &a,
                            float *partial, cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return tc_forward_layer_impl<64>(ctx, csr, a, partial, st);
    case 128: return tc_forward_layer_impl<128>(ctx, csr, a, partial, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

}  // namespace occu
