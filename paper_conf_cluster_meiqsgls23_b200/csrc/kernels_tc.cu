// Tensor-core (tcgen05) forward GEMM kernels of the FP32 path, sm_100a.
//
// The three dense contractions of an ANEE layer — h W_uᵀ (P141), W_e e (P145),
// W_m e' (P149) — run in one warp-specialised, software-pipelined kernel
// template `rowgemm_kernel<D, EPI>` with a fused row-wise epilogue:
//   EPI_NODE : h̄ = LReLU(.), p = h̄·a_s, q = h̄·a_d                    (a2)
//   EPI_EDGE : e' = σ((p[s] + q[t]) · .)                              (a3)
//   EPI_GATE : g = softmax over the D channels of (.)                 (a4)
// followed by the CUDA-core gather + segmented sum (a5, a6, kernels_simt.cu).
//
// FP32 accuracy from 16-bit tensor cores ("fp16x2 split"): every
// input row x is scaled by a power of two 2^e_r (row max -> [2^14, 2^15)),
// every weight matrix by 2^f, and split x = x0 + x1, w = w0 + w1 with
// x0 = fp16(x), x1 = fp16(x - x0) (22 significant bits together).  The MMA
// accumulates x0·w0 + x0·w1 + x1·w0 in FP32 (TMEM); the dropped x1·w1 term is
// ~2^-22 relative.  The epilogue multiplies by 2^-(e_r + f), which is exact.
//
// CTA = 26 warps (NTH = 832), persistent over 128-row tiles, 1 CTA per SM:
//   warp 0       producer: bulk copy of the weight images, then 2D TMA loads (128 rows x 32
//                fp32 SW128 boxes, OOB rows zero-filled) of the next tiles into a 2-slot ring;
//   warp 1       TMEM allocator + MMA issuer: 3·K/16 tcgen05.mma (M=128, N=D, K=16, A from
//                TMEM, B = SW128 K-major weight images in smem), commit -> accumulator-full /
//                A-free mbarriers;
//   warps 2-9    converters, thread = (row, K-half): per-row power-of-two scale (row max
//                exchanged between the halves), fp16x2 split into TMEM A[i%2] (tcgen05.st);
//   warps 10-25  epilogue, two groups of 8 warps on alternating tiles (two warps per TMEM lane
//                quarter, one per column half): tcgen05.ld of ACC[i%2], the fused row epilogue,
//                coalesced stores through per-warp transpose buffers.
// TMEM: A[2] x 128 columns + ACC[2] x 128 columns = 512.  Loads of tile i+1, the MMAs of
// tile i and the epilogues of tiles i-1, i-2 overlap.
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>
#include <vector>

#include "occu_internal.h"
#include "tc_common.cuh"

namespace occu {
namespace {

constexpr int TM = 128;
constexpr int NTH = 832;          // warp 0 producer, 1 MMA, 2-9 converters, 10-25 epilogue
constexpr int EPI0 = 10;          // first epilogue warp
constexpr uint32_t TMEM_COLS = 512;
constexpr int EPI_NODE = 0, EPI_EDGE = 1, EPI_GATE = 2;
// backward epilogues (SURVEY §8(c) step BW)
constexpr int EPI_PLAIN = 3;      // out = acc (+ add)
constexpr int EPI_GATEBWD = 4;    // g = softmax(acc); dm = dA[t]; MG = dm ⊙ g; DV = g ⊙ (dm ⊙ h̄[s] - <g, dm ⊙ h̄[s]>)
constexpr int EPI_EDGEBWD = 5;    // z = acc; dy = de ⊙ e' ⊙ σ(-αz); dα = <dy, z>; DZ = α dy
constexpr int EPI_GATEAGG = 6;

#ifdef OCCU_TC_TIMING
// Per-role busy/wait cycle counters of CTA 0 (debug builds only).
__device__ unsigned long long g_tc_time[32][4];
#define TT_DECL unsigned long long tt_w = 0, tt_b = 0, tt_0 = clock64(), tt_1;
#define TT_WAIT_BEGIN tt_1 = clock64(); tt_b += tt_1 - tt_0;
#define TT_WAIT_END tt_0 = clock64(); tt_w += tt_0 - tt_1;
#define TT_FLUSH(slot)                                                            \
  do {                                                                            \
    tt_b += clock64() - tt_0;                                                     \
    if (blockIdx.x == 0 && (threadIdx.x & 31) == 0) {                             \
      g_tc_time[slot][0] += tt_w; g_tc_time[slot][1] += tt_b; g_tc_time[slot][2] += 1; \
    }                                                                             \
  } while (0)
__device__ unsigned long long g_eg_time[32][4];
#define TT_FLUSH_EG(slot)                                                         \
  do {                                                                            \
    tt_b += clock64() - tt_0;                                                     \
    if (blockIdx.x == 0 && (threadIdx.x & 31) == 0) {                             \
      g_eg_time[slot][0] += tt_w; g_eg_time[slot][1] += tt_b; g_eg_time[slot][2] += 1; \
    }                                                                             \
  } while (0)
#else
#define TT_DECL
#define TT_WAIT_BEGIN
#define TT_WAIT_END
#define TT_FLUSH(slot)
#define TT_FLUSH_EG(slot)
#endif    // g = softmax(acc); m = g ⊙ h̄[s]; h[t] = LReLU(Σ_seg m) (a4-a6 fused)



__device__ __forceinline__ uint32_t a_col(int j) { return uint32_t(j) * 128u; }
__device__ __forceinline__ uint32_t acc_col(int j) { return 256u + uint32_t(j) * 128u; }
__device__ __forceinline__ float lrelu(float x, float s) { return x > 0.f ? x : s * x; }
// Fast exp / reciprocal (MUFU.EX2 / MUFU.RCP, ~2^-22 relative): exact at the
// closed-form special cases used by the bit-exact tests (exp(0) = 1, 1/2^k).
constexpr float LOG2E = 1.4426950408889634f;
__device__ __forceinline__ float ex2(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float fast_exp(float x) { return ex2(x * LOG2E); }
__device__ __forceinline__ float fast_rcp(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

struct RowGemmArgs {
  const float *A;          // [R][K] input rows (fp32)
  int K, R;
  const float *W;          // [D][K] (unused by the kernel: see wimg)
  const uint8_t *wimg;     // prebuilt fp16x2 SW128 images of W: [w0 | w1], Kpad*D*2 bytes each
  const int *wfexp;        // weight scale exponent f
  float *out;              // [R][D]
  const float *a_s, *a_d;  // NODE
  float *p, *q;            // NODE outputs
  const float *pin, *qin;  // EDGE: p, q of the layer
  const int32_t *src, *dst;
  float slope;
  int transW;              // W given as [K][D] (the row-GEMM uses its transpose)
  const float *add;        // PLAIN: [R][D] addend (nullable)
  float *out2;             // GATEBWD: DV
  const float *dh, *h, *hbar, *e, *de;
  const float *mask_h;     // PLAIN: multiply row by LReLU'(mask_h row) (÷ deg for MEAN) -> dA
  int mask_bf;             // mask_h rows are BF16 (OCCU_BF16 training)
  const uint32_t *mask_bits;   // PLAIN: the mask's sign bits [R][D/32] (word c, bit l: channel V·l + c)
                               // instead of mask_h rows (gather_segsum's training output)
  const float *bias;       // PLAIN: per-column bias (nullable), then ReLU if relu
  int relu;
  const int32_t *in_ptr;
  int mean;
  float *dal;              // EDGEBWD: dα [R]
  float *part;             // GATEAGG: [R/32 units][2 slots][D] boundary-segment partials
  int rev;                 // walk tiles last-to-first (reads what the previous kernel wrote last, still in L2)
  const int *rexp;         // d = 256 NODE: per-row scale exponents (row_exp_kernel)
  int dot2;                // EDGEBWD: dα by the compensated FP32 dot (else float64 FMA)
  int *out_rexp;           // EDGEBWD: scale exponents of the output rows (for the next row-GEMM)
};

struct Smem {
  uint8_t *w0, *w1;
  float *slot0;
  int slot_floats;
  __device__ __forceinline__ float *slot(int j) const { return slot0 + j * slot_floats; }
  uint64_t *full, *empty, *afull, *afree, *accfull, *accfree, *eready, *wfull;
  uint32_t *tmem_slot;
  int *fexp;
  float *red;
  float *avec;             // [2*D] a_s, a_d (NODE)
  int *erow;               // [4][128] per-row scale exponents, converter -> epilogue
  float *xbuf;             // per worker warp: 8 x 36 floats (coalescing transpose)
  float *xch;              // [2 groups][2 values][2 halves][128 rows] row-partial exchange
};

__host__ __device__ inline int kpad_of(int K) { return (K + 63) / 64 * 64; }
// input slot: ceil(K/32) TMA boxes of 128 rows x 32 fp32 (128 B, SW128-swizzled)
__host__ __device__ inline int nbox_of(int K) { return (K + 31) / 32; }
__host__ __device__ inline size_t smem_bytes(int D, int K) {
  const size_t img = size_t(kpad_of(K)) * D * 2;
  const size_t slot = size_t(nbox_of(K)) * 16384;
  return 1024 + 2 * img + 2 * slot + 4096 + 16 * 16 * 20 * 4 + 2 * 2 * 2 * 128 * 4 + 2 * 128 * 4;
}

__device__ __forceinline__ Smem carve(uint8_t *raw, int D, int K) {
  Smem s;
  const uint32_t a = tc::smem_u32(raw);
  uint8_t *base = raw + ((1024 - (a & 1023)) & 1023);
  const size_t img = size_t(kpad_of(K)) * D * 2;
  const size_t slot = size_t(nbox_of(K)) * 16384;
  s.w0 = base;
  s.w1 = base + img;
  s.slot0 = reinterpret_cast<float *>(base + 2 * img);
  s.slot_floats = int(slot / 4);
  uint8_t *misc = base + 2 * img + 2 * slot;
  uint64_t *bars = reinterpret_cast<uint64_t *>(misc);
  s.full = bars;
  s.empty = bars + 2;
  s.afull = bars + 4;
  s.afree = bars + 6;
  s.accfull = bars + 8;
  s.accfree = bars + 10;
  s.eready = bars + 12;                 // 4
  s.wfull = bars + 16;
  s.tmem_slot = reinterpret_cast<uint32_t *>(misc + 144);
  s.fexp = reinterpret_cast<int *>(misc + 148);
  s.red = reinterpret_cast<float *>(misc + 256);
  s.avec = reinterpret_cast<float *>(misc + 512);
  s.erow = reinterpret_cast<int *>(misc + 1536);
  s.xbuf = reinterpret_cast<float *>(misc + 4096);
  s.xch = s.xbuf + 16 * 16 * 20;
  return s;
}

// e such that max|x|·2^e lies in [2^14, 2^15); 0 for an all-zero row.  Capped at 100 so that
// 2^e stays finite and the epilogue's 2^-(e_row + f) (f <= ~30 for the weights) stays a
// representable power of two: a row whose largest entry is below 2^-86 keeps less than 22
// significant bits in fp16x2, an absolute error below 2^-108 (without the cap 2^e overflowed
// to inf and such rows came out NaN — seen on tiny gradient rows under reading B + MEAN).
__device__ __forceinline__ int scale_exp(float mx) { return occu_row_scale_exp(mx); }

// x (already scaled) -> packed fp16 pair hi and lo for elements (v0, v1).
__device__ __forceinline__ void split2(float v0, float v1, uint32_t &hi, uint32_t &lo) {
  const __half2 h = __floats2half2_rn(v0, v1);
  const float2 f = __half22float2(h);
  const __half2 l = __floats2half2_rn(v0 - f.x, v1 - f.y);
  hi = *reinterpret_cast<const uint32_t *>(&h);
  lo = *reinterpret_cast<const uint32_t *>(&l);
}

// Coalesced store of a 32-column chunk of the warp's 32 rows (thread = row):
// rows are transposed through an 8 x 36 per-warp buffer so that each warp store
// instruction writes 4 full 128-byte lines instead of 32 partial ones.
template <int D>
__device__ __forceinline__ void warp_store_chunk(float *buf, float *__restrict__ out, long wrow0,
                                                 int wrows, int c0, const float (&v)[16], int lane) {
  // 16 columns (64 B) per row; two 16-row passes through a 16 x 20 buffer
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    if ((lane >> 4) == h) {
      float *b = buf + (lane & 15) * 20;
#pragma unroll
      for (int u = 0; u < 16; u += 4)
        *reinterpret_cast<float4 *>(b + u) = make_float4(v[u], v[u + 1], v[u + 2], v[u + 3]);
    }
    __syncwarp();
#pragma unroll
    for (int it = 0; it < 2; ++it) {
      const int idx = it * 32 + lane, r = idx >> 2, c4 = (idx & 3) * 4;
      const int rr = h * 16 + r;
      if (rr < wrows)
        *reinterpret_cast<float4 *>(out + (wrow0 + rr) * D + c0 + c4) =
            *reinterpret_cast<const float4 *>(buf + r * 20 + c4);
    }
    __syncwarp();
  }
}

__device__ __forceinline__ int tile_of(const RowGemmArgs &a, int tiles, int i) {
  const int t = int(blockIdx.x) + i * int(gridDim.x);
  return a.rev ? tiles - 1 - t : t;
}

__device__ __forceinline__ void group_bar(int g) {
  asm volatile("bar.sync %0, 256;" ::"r"(1 + g) : "memory");
}

// float4 of row r, columns [k, k+4) (k % 4 == 0) inside a slot of SW128 TMA boxes.
__device__ __forceinline__ float4 slot_ld4(const float *slot, int r, int k) {
  const int b = k >> 5, c = (k & 31) >> 2;
  return *reinterpret_cast<const float4 *>(slot + b * 4096 + r * 32 + ((c ^ (r & 7)) << 2));
}

template <int D, int EPI>
__global__ void __launch_bounds__(NTH, 1) rowgemm_kernel(const __grid_constant__ CUtensorMap tmap,
                                                         RowGemmArgs a) {
  extern __shared__ uint8_t smem_raw[];
#ifdef OCCU_TC_TIMING
  const unsigned long long t_entry = clock64();
#endif
  const int K = a.K, Kpad = kpad_of(K), NB = nbox_of(K);
  Smem s = carve(smem_raw, D, K);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  pdl_trigger();
  if (threadIdx.x == 0) {
    for (int j = 0; j < 2; ++j) {
      tc::mbar_init(s.full + j, 1);
      tc::mbar_init(s.empty + j, 256);
      tc::mbar_init(s.afull + j, 256);
      tc::mbar_init(s.afree + j, 1);
      tc::mbar_init(s.accfull + j, 1);
      tc::mbar_init(s.accfree + j, 256);
    }
    for (int j = 0; j < 4; ++j) tc::mbar_init(s.eready + j, 256);
    tc::mbar_init(s.wfull, 1);
    tc::fence_mbar_init();
  }
  if (warp == 1) tc::tmem_alloc<TMEM_COLS>(s.tmem_slot);
  pdl_wait();                              // predecessor's writes visible from here on
  // ---- weights: prebuilt fp16x2 images (wimage_kernel), bulk-copied by the producer ----
  const int fexp = __ldg(a.wfexp);
  const bool noshift = __ldg(a.wfexp + 1) != 0;
  if (EPI == EPI_NODE)
    for (int i = threadIdx.x; i < D; i += NTH) {
      s.avec[i] = a.a_s[i];
      s.avec[D + i] = a.a_d[i];
    }
  // generic-proxy smem writes (weight images) must be visible to the async proxy (MMA)
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  const uint32_t tmem = *s.tmem_slot;
#ifdef OCCU_TC_TIMING
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    g_tc_time[30][1] += clock64() - t_entry;
    g_tc_time[30][2] += 1;
  }
#endif

  const int tiles = (a.R + TM - 1) / TM;
  const int my = blockIdx.x < tiles ? (tiles - 1 - int(blockIdx.x)) / int(gridDim.x) + 1 : 0;

  if (warp == 0) {
    // ---------------- producer: tile i -> slot i%2 (TMA 2D, OOB rows zero-filled) -------
    if (lane == 0) {
      TT_DECL
      tc::prefetch_tmap(&tmap);
      {   // weight images -> smem (16 KB bulk copies)
        const uint32_t ib = uint32_t(Kpad) * D * 2;
        tc::mbar_arrive_expect_tx(s.wfull, 2 * ib);
        for (uint32_t o = 0; o < ib; o += 16384) {
          const uint32_t n = ib - o < 16384 ? ib - o : 16384;
          tc::bulk_g2s(s.w0 + o, a.wimg + o, n, s.wfull);
          tc::bulk_g2s(s.w1 + o, a.wimg + ib + o, n, s.wfull);
        }
      }
      for (int i = 0; i < my; ++i) {
        const int j = i & 1;
        const int r0 = tile_of(a, tiles, i) * TM;
        TT_WAIT_BEGIN
        if (i >= 2) tc::mbar_wait(s.empty + j, ((i >> 1) - 1) & 1);
        TT_WAIT_END
        tc::mbar_arrive_expect_tx(s.full + j, uint32_t(NB) * 16384u);
        for (int b = 0; b < NB; ++b) tc::tma_load_2d(s.slot(j) + b * 4096, &tmap, 32 * b, r0, s.full + j);
      }
      TT_FLUSH(0);
    }
    __syncwarp();
  } else if (warp == 1) {
    // ---------------- MMA issuer: A[i%2] -> ACC[i%2] ----------------
    TT_DECL
    const uint32_t idsc = tc::idesc(128, uint32_t(D), tc::FMT_F16);
    const uint32_t w0a = tc::smem_u32(s.w0), w1a = tc::smem_u32(s.w1);
    const int nk = (K + 15) / 16;
    tc::mbar_wait(s.wfull, 0);
    for (int i = 0; i < my; ++i) {
      const int j = i & 1;
      TT_WAIT_BEGIN
      tc::mbar_wait(s.afull + j, (i >> 1) & 1);
      if (i >= 2) tc::mbar_wait(s.accfree + j, ((i >> 1) - 1) & 1);
      TT_WAIT_END
      tc::fence_after_sync();
      if (lane == 0) {
        const uint32_t d = tmem + acc_col(j);
        for (int kk = 0; kk < nk; ++kk) {
          const uint32_t boff = uint32_t(kk >> 2) * uint32_t(D) * 128u + uint32_t(kk & 3) * 32u;
          const uint64_t b0 = tc::sdesc_sw128(w0a + boff), b1 = tc::sdesc_sw128(w1a + boff);
          const uint32_t a0 = tmem + a_col(j) + uint32_t(kk) * 8u;
          const uint32_t a1 = a0 + uint32_t(Kpad / 2);
          tc::mma_f16_ts(d, a0, b0, idsc, kk > 0 ? 1u : 0u);
          tc::mma_f16_ts(d, a0, b1, idsc, 1u);
          tc::mma_f16_ts(d, a1, b0, idsc, 1u);
        }
        tc::mma_commit(s.accfull + j);
        tc::mma_commit(s.afree + j);
      }
      __syncwarp();
    }
    TT_FLUSH(1);
  } else if (warp < EPI0) {
    // ---------------- converters (warps 2-9): thread = (row, K-half) -> TMEM A ----------------
    // Input rows of the node transform (h) get a per-row power-of-two scale from the row max
    // (exchanged between the two K-halves); edge states e' lie in [0, 1] and are split
    // unscaled (fp16 normal down to 2^-14; below that the absolute error stays < 2^-25,
    // which is what matters where e' is consumed).
    const int qd = warp & 3;
    const int kh = (warp - 2) >> 2;
    const int row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    const int KH = Kpad / 2;                       // K-elements per half
    const int kb = kh * KH, ke = min(K, kb + KH);
    float *cmax = s.xch + 2 * 2 * 2 * 128;         // [2 halves][128 rows]
    TT_DECL
    for (int i = 0; i < my; ++i) {
      const int j = i & 1;
      const long r0 = long(tile_of(a, tiles, i)) * TM;
      const bool live = row < min(TM, int(a.R - r0));
      // PLAIN with handed-over exponents: the row's exponent is requested before the waits
      const int er_pre = (EPI == EPI_PLAIN && a.rexp && live) ? __ldg(a.rexp + r0 + row) : 0;
      TT_WAIT_BEGIN
      tc::mbar_wait(s.full + j, (i >> 1) & 1);
      if (i >= 2) tc::mbar_wait(s.afree + j, ((i >> 1) - 1) & 1);
      TT_WAIT_END
      const float *sl = s.slot(j);
      int er = 0;                                  // e' in [0, 1]: no scaling (see above)
      if (EPI == EPI_PLAIN && a.rexp) {
        er = er_pre;                               // handed over by the rows' producer
      } else if (EPI == EPI_NODE || EPI == EPI_PLAIN) {
        float mx = 0.f;
        if (live)
#pragma unroll 4
          for (int k = kb; k < ke; k += 4) {
            const float4 v = slot_ld4(sl, row, k);
            mx = fmaxf(mx, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w))));
          }
        cmax[kh * 128 + row] = mx;
        asm volatile("bar.sync 3, 256;" ::: "memory");
        mx = fmaxf(mx, cmax[(kh ^ 1) * 128 + row]);
        er = scale_exp(mx);
        asm volatile("bar.sync 3, 256;" ::: "memory");   // cmax reused next tile
      }
      const float xs = ldexpf(1.f, er);
      for (int c0 = 0; c0 < KH / 2; c0 += 16) {
        uint32_t x0[16], x1[16];
#pragma unroll
        for (int u = 0; u < 16; u += 2) {
          const int k = kb + 2 * (c0 + u);
          float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
          if (live && k < K) v = slot_ld4(sl, row, k);
          if (EPI == EPI_NODE || EPI == EPI_PLAIN) {
            v.x *= xs; v.y *= xs; v.z *= xs; v.w *= xs;
          }
          split2(v.x, v.y, x0[u], x1[u]);
          split2(v.z, v.w, x0[u + 1], x1[u + 1]);
        }
        const uint32_t col = a_col(j) + uint32_t(kb / 2 + c0);
        tc::tmem_st16(lane_base + col, x0);
        tc::tmem_st16(lane_base + col + Kpad / 2, x1);
      }
      if (kh == 0) s.erow[(i & 3) * 128 + row] = er;
      tc::tmem_st_wait();
      tc::fence_before_sync();
      tc::mbar_arrive(s.empty + j);
      tc::mbar_arrive(s.afull + j);
      tc::mbar_arrive(s.eready + (i & 3));
    }
    TT_FLUSH(2 + (warp - 2));
  } else {
    // ---------------- epilogue: two groups of 8 warps (6-13, 14-21) -----------------
    // group g handles tiles i = g, g+2, ... from ACC[g]; a row is shared by two warps of
    // the same TMEM lane quarter: half hf owns output columns [hf*D/2, (hf+1)*D/2).
    const int wi = warp - EPI0;
    const int g = wi >> 3;
    const int hf = (wi >> 2) & 1;
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    float *xg = s.xch + g * (2 * 2 * 128);           // [value][half][row]
    float *wbuf = s.xbuf + wi * (16 * 20);
    constexpr int DH = D / 2;
    const int cb = hf * DH;
    TT_DECL
    for (int i = g; i < my; i += 2) {
      const int j = i & 1;
      const long r0 = long(tile_of(a, tiles, i)) * TM;
      const int nrows = min(TM, int(a.R - r0));
      const bool live = row < nrows;
      float aux = 0.f;
      if ((EPI == EPI_EDGE || EPI == EPI_EDGEBWD) && hf == 0 && live)
        aux = __ldg(a.pin + __ldg(a.src + r0 + row)) + __ldg(a.qin + __ldg(a.dst + r0 + row));  // α (R1)
      // EDGEBWD: the row's first de chunk is fetched before waiting on the accumulator, and
      // every later chunk one step ahead (the epilogue is paced by these per-row loads)
      // PLAIN: likewise the row's addend (or, without one, its FP32 mask) — the one per-row
      // stream of the de / dh_prev GEMMs — one chunk ahead
      float4 dpre[4];
      const float *pre_src = EPI == EPI_EDGEBWD ? a.de
                           : (EPI == EPI_PLAIN ? (a.add ? a.add : ((a.mask_bf || a.mask_bits) ? nullptr : a.mask_h)) : nullptr);
      // PLAIN with sign bits: the row's D/32 mask words (16 B at D = 128) instead of a D-float row
      constexpr int MV = D / 32;
      uint32_t mw[EPI == EPI_PLAIN ? MV : 1];
      if (EPI == EPI_PLAIN) {
#pragma unroll
        for (int c = 0; c < (EPI == EPI_PLAIN ? MV : 1); ++c)
          mw[c] = (a.mask_bits && live) ? __ldg(a.mask_bits + (r0 + row) * MV + c) : 0u;
      }
      if (EPI == EPI_EDGEBWD || EPI == EPI_PLAIN) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
          dpre[u] = (live && pre_src) ? __ldg(reinterpret_cast<const float4 *>(pre_src + (r0 + row) * D + hf * (D / 2) + 4 * u))
                                      : make_float4(0.f, 0.f, 0.f, 0.f);
      }
      TT_WAIT_BEGIN
      tc::mbar_wait(s.eready + (i & 3), (i >> 2) & 1);
      const int er = s.erow[(i & 3) * 128 + row];
      tc::mbar_wait(s.accfull + j, (i >> 1) & 1);
      TT_WAIT_END
      tc::fence_after_sync();
      if (EPI == EPI_EDGE || EPI == EPI_EDGEBWD) {
        if (hf == 0) xg[row] = aux;
        group_bar(g);
        aux = xg[row];
      }
      const float un = ldexpf(1.f, -(er + fexp));
      const long grow = r0 + row;
      const long wrow0 = r0 + qd * 32;
      const int wrows = max(0, min(32, nrows - qd * 32));
      const uint32_t acc = lane_base + acc_col(j) + cb;
      if (EPI == EPI_PLAIN) {
        const bool pre_add = a.add != nullptr;                 // dpre holds the addend chunk
        const bool pre_mask = !pre_add && pre_src != nullptr;  // dpre holds the FP32 mask chunk
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          float4 dcur[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) dcur[u] = dpre[u];
          if (pre_src && c0 + 16 < DH) {
            const float *pn = pre_src + grow * D + cb + c0 + 16;
#pragma unroll
            for (int u = 0; u < 4; ++u)
              dpre[u] = live ? __ldg(reinterpret_cast<const float4 *>(pn + 4 * u)) : make_float4(0.f, 0.f, 0.f, 0.f);
          }
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = __uint_as_float(r[u]) * un;
          if (a.mask_bits && live) {
            float dsc = 1.f;
            if (a.mean) {
              const int deg = __ldg(a.in_ptr + grow + 1) - __ldg(a.in_ptr + grow);
              dsc = float(deg > 0 ? deg : 1);
            }
            const int sh = (cb + c0) / MV;                 // cb + c0 is a multiple of 16 (and of MV)
#pragma unroll
            for (int u = 0; u < 16; ++u) {
              o[u] *= ((mw[u % MV] >> (sh + u / MV)) & 1u) ? 1.f : a.slope;
              if (a.mean) o[u] = o[u] / dsc;
            }
          } else if (a.mask_h && live) {
            const float *mr = a.mask_h + grow * D + cb + c0;
            const uint16_t *mb = reinterpret_cast<const uint16_t *>(a.mask_h) + grow * D + cb + c0;
            float dsc = 1.f;
            if (a.mean) {
              const int deg = __ldg(a.in_ptr + grow + 1) - __ldg(a.in_ptr + grow);
              dsc = float(deg > 0 ? deg : 1);
            }
#pragma unroll
            for (int u = 0; u < 16; u += 4) {
              float4 x;
              if (a.mask_bf) {      // only the sign matters: BF16 keeps it
                const uint2 b = __ldg(reinterpret_cast<const uint2 *>(mb + u));
                x = make_float4(__uint_as_float(b.x << 16), __uint_as_float(b.x & 0xFFFF0000u),
                                __uint_as_float(b.y << 16), __uint_as_float(b.y & 0xFFFF0000u));
              } else if (pre_mask) {
                x = dcur[u >> 2];
              } else {
                x = __ldg(reinterpret_cast<const float4 *>(mr + u));
              }
              const float xv[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
              for (int t = 0; t < 4; ++t) {
                o[u + t] *= xv[t] > 0.f ? 1.f : a.slope;
                if (a.mean) o[u + t] = o[u + t] / dsc;
              }
            }
          }
          if (a.bias) {
#pragma unroll
            for (int u = 0; u < 16; ++u) {
              o[u] += __ldg(a.bias + cb + c0 + u);
              if (a.relu) o[u] = fmaxf(o[u], 0.f);
            }
          }
          if (pre_add && live) {
#pragma unroll
            for (int u = 0; u < 16; u += 4) {
              const float4 x = dcur[u >> 2];
              o[u] += x.x; o[u + 1] += x.y; o[u + 2] += x.z; o[u + 3] += x.w;
            }
          }
          warp_store_chunk<D>(wbuf, a.out, wrow0, wrows, cb + c0, o, lane);
        }
      } else if (EPI == EPI_EDGEBWD) {
        // dα = <dy, z> needs more than FP32 (cancellation): compensated FP32 dot (Ogita-Rump-
        // Oishi Dot2: TwoProduct by FMA + TwoSum, as accurate as a 2x-precision sum rounded
        // once) — 9 FP32 operations per element instead of two F2F.F64 conversions and a DFMA
        double dpart = 0.0;
        float ds = 0.f, dc = 0.f;
        float omax = 0.f;                            // max |DZ| of the row half (out_rexp)
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
          float4 dcur[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) dcur[u] = dpre[u];
          if (c0 + 16 < DH) {
            const float *dn = a.de + grow * D + cb + c0 + 16;
#pragma unroll
            for (int u = 0; u < 4; ++u)
              dpre[u] = live ? __ldg(reinterpret_cast<const float4 *>(dn + 4 * u)) : make_float4(0.f, 0.f, 0.f, 0.f);
          }
          const float cexp = -aux * un * LOG2E;
#pragma unroll
          for (int u = 0; u < 16; u += 4) {
            float4 ev = make_float4(0.f, 0.f, 0.f, 0.f);
            const float4 dv = dcur[u >> 2];
            // e' = σ(αz) is recomputed from the accumulator exactly as EPI_EDGE formed it
            // (same rows, weight images and MMA order -> same bits) unless a.e is given
            if (live && a.e) ev = __ldg(reinterpret_cast<const float4 *>(a.e + grow * D + cb + c0 + u));
            float evv[4] = {ev.x, ev.y, ev.z, ev.w};
            const float dvv[4] = {dv.x, dv.y, dv.z, dv.w};
            float sneg[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              // τ = e^{-y}, y = α z: σ(y) = 1/(1 + τ) (the forward's e', same bits) and
              // σ(-y) = τ·σ(y) — one MUFU ex2 + one rcp per element; τ = inf -> σ(-y) = 1
              const float tau = ex2(__uint_as_float(r[u + t]) * cexp);
              const float sp = fast_rcp(1.f + tau);
              if (!a.e) evv[t] = sp;
              sneg[t] = tau < 3.0e38f ? tau * sp : 1.f;
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              const float z = __uint_as_float(r[u + t]) * un;
              // σ'(y) = σ(y)·σ(-y), y = α z (recomputed): no 1 - e' cancellation
              const float dy = dvv[t] * evv[t] * sneg[t];
              if (a.dot2) {
                const float pr = dy * z, pe = fmaf(dy, z, -pr);          // TwoProduct
                const float t1 = ds + pr, bp = t1 - ds;                  // TwoSum(ds, pr)
                const float se = (ds - (t1 - bp)) + (pr - bp);
                ds = t1;
                dc += se + pe;
              } else {
                dpart = fma(double(dy), double(z), dpart);
              }
              o[u + t] = aux * dy;
              omax = fmaxf(omax, fabsf(o[u + t]));
            }
          }
          warp_store_chunk<D>(wbuf, a.out, wrow0, wrows, cb + c0, o, lane);
        }
        double *xd = reinterpret_cast<double *>(xg);   // reuses the whole exchange area
        if (a.dot2) dpart = double(ds) + double(dc);
        group_bar(g);                                   // everyone has consumed the α slot
        xd[hf * 128 + row] = dpart;
        group_bar(g);
        if (hf == 0 && live) a.dal[grow] = float(dpart + xd[128 + row]);
        if (a.out_rexp) {                               // the row's max |DZ| -> its fp16x2 exponent
          group_bar(g);                                 // xd consumed
          xg[hf * 128 + row] = omax;
          group_bar(g);
          if (hf == 0 && live) a.out_rexp[grow] = scale_exp(fmaxf(omax, xg[128 + row]));
        }
      } else if (EPI == EPI_GATEBWD) {
        // softmax statistics (as the forward gate)
        float m = -INFINITY;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) m = fmaxf(m, __uint_as_float(r[u]) * un);
        }
        xg[hf * 128 + row] = m;
        group_bar(g);
        m = fmaxf(m, xg[(hf ^ 1) * 128 + row]);
        float sum = 0.f;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) sum += fast_exp(__uint_as_float(r[u]) * un - m);
        }
        xg[256 + hf * 128 + row] = sum;
        group_bar(g);
        sum = hf == 0 ? sum + xg[256 + 128 + row] : xg[256 + row] + sum;
        const float inv = fast_rcp(sum);
        // dA[t] = dh[t] ⊙ LReLU'(h[t]) (÷ deg for MEAN); gathers by destination / source
        const int tn = live ? __ldg(a.dst + grow) : 0;
        const int sn = live ? __ldg(a.src + grow) : 0;
        float dscale = 1.f;
        const bool is_dA = a.h == nullptr;
        if (!is_dA && a.mean && live) {
          const int deg = __ldg(a.in_ptr + tn + 1) - __ldg(a.in_ptr + tn);
          dscale = float(deg > 0 ? deg : 1);
        }
        const float *dhr = a.dh + long(tn) * D + cb, *hr = is_dA ? dhr : a.h + long(tn) * D + cb;
        const float *hbr = a.hbar + long(sn) * D + cb;
        double dotd = 0.0;     // <g, dg> in float64 (cancellation)
        float dot = 0.f;
        group_bar(g);          // everyone has read the (m, sum) exchange slots
#pragma unroll 1
        for (int pass = 0; pass < 2; ++pass) {
#pragma unroll 1
          for (int c0 = 0; c0 < DH; c0 += 16) {
            uint32_t r[16];
            tc::tmem_ld16(acc + c0, r);
            tc::tmem_ld_wait();
            float o[16];
#pragma unroll
            for (int u = 0; u < 16; u += 4) {
              float4 d4 = make_float4(0.f, 0.f, 0.f, 0.f), h4 = d4, b4 = d4;
              if (live) {
                d4 = __ldg(reinterpret_cast<const float4 *>(dhr + c0 + u));
                if (!is_dA) h4 = __ldg(reinterpret_cast<const float4 *>(hr + c0 + u));
                b4 = __ldg(reinterpret_cast<const float4 *>(hbr + c0 + u));
              }
              const float dv[4] = {d4.x, d4.y, d4.z, d4.w}, hv[4] = {h4.x, h4.y, h4.z, h4.w};
              const float bv[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
              for (int t = 0; t < 4; ++t) {
                const float gg = fast_exp(__uint_as_float(r[u + t]) * un - m) * inv;
                float dm = dv[t];
                if (!is_dA) {
                  dm = dm * (hv[t] > 0.f ? 1.f : a.slope);
                  if (a.mean) dm = dm / dscale;
                }
                const float dg = dm * bv[t];
                if (pass == 0) {
                  dotd = fma(double(gg), double(dg), dotd);
                  o[u + t] = dm * gg;                              // MG
                } else {
                  o[u + t] = gg * (dg - dot);                      // DV
                }
              }
            }
            warp_store_chunk<D>(wbuf, pass == 0 ? a.out : a.out2, wrow0, wrows, cb + c0, o, lane);
          }
          if (pass == 0) {
            double *xd = reinterpret_cast<double *>(xg);
            xd[hf * 128 + row] = dotd;
            group_bar(g);
            dot = float(hf == 0 ? dotd + xd[128 + row] : xd[row] + dotd);   // fixed order
          }
        }
      } else if (EPI == EPI_GATEAGG) {
        float m = -INFINITY;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) m = fmaxf(m, __uint_as_float(r[u]) * un);
        }
        xg[hf * 128 + row] = m;
        group_bar(g);
        m = fmaxf(m, xg[(hf ^ 1) * 128 + row]);
        float sum = 0.f;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) sum += fast_exp(__uint_as_float(r[u]) * un - m);
        }
        xg[256 + hf * 128 + row] = sum;
        group_bar(g);
        sum = hf == 0 ? sum + xg[256 + 128 + row] : xg[256 + row] + sum;
        const float inv = fast_rcp(sum);
        // destination segments inside this warp's 32 consecutive (dst-sorted) edges
        const int tn = live ? __ldg(a.dst + grow) : -1 - lane;         // pad rows: own segment
        const int sn = live ? __ldg(a.src + grow) : 0;
        const int tprev = __shfl_up_sync(0xffffffffu, tn, 1);
        const int tnext = __shfl_down_sync(0xffffffffu, tn, 1);
        const bool head = lane == 0 || tprev != tn;
        const bool tail = lane == 31 || tnext != tn;
        const unsigned heads = __ballot_sync(0xffffffffu, head);
        const int start = 31 - __clz(heads & (0xffffffffu >> (31 - lane)));
        const int maxlen = __reduce_max_sync(0xffffffffu, unsigned(lane - start + 1));
        int beg = 0, end = 0;
        if (tail && live) {
          beg = __ldg(a.in_ptr + tn);
          end = __ldg(a.in_ptr + tn + 1);
        }
        const bool before = live && beg < wrow0 + start;               // segment began earlier
        const bool after = live && end > wrow0 + lane + 1;               // continues after this warp
        float dsc = 1.f;
        if (a.mean) dsc = float(end - beg > 0 ? end - beg : 1);
        const float *hbr = a.hbar + long(sn) * D + cb;
        const long unit = wrow0 >> 5;
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float v[16];
#pragma unroll
          for (int u = 0; u < 16; u += 4) {
            float4 b4 = make_float4(0.f, 0.f, 0.f, 0.f);
            if (live) b4 = __ldg(reinterpret_cast<const float4 *>(hbr + c0 + u));
            const float bv[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
            for (int t = 0; t < 4; ++t)
              v[u + t] = fast_exp(__uint_as_float(r[u + t]) * un - m) * inv * bv[t];   // m = g ⊙ h̄[s]
          }
          // segmented inclusive scan across lanes (fixed tree order)
          for (int d = 1; d < maxlen; d <<= 1) {        // only as many steps as the longest run
#pragma unroll
            for (int u = 0; u < 16; ++u) {
              const float o = __shfl_up_sync(0xffffffffu, v[u], d);
              if (lane - d >= start) v[u] += o;
            }
          }
          if (tail && live) {
            if (!before && !after) {                                   // complete segment
              float *hr = a.out + long(tn) * D + cb + c0;
#pragma unroll
              for (int u = 0; u < 16; u += 4) {
                float o4[4];
#pragma unroll
                for (int t = 0; t < 4; ++t) {
                  float x = v[u + t];
                  if (a.mean) x = x / dsc;
                  o4[t] = lrelu(x, a.slope);
                }
                *reinterpret_cast<float4 *>(hr + u) = make_float4(o4[0], o4[1], o4[2], o4[3]);
              }
            } else {
              float *pr = a.part + (unit * 2 + (before ? 0 : 1)) * D + cb + c0;
#pragma unroll
              for (int u = 0; u < 16; u += 4)
                *reinterpret_cast<float4 *>(pr + u) = make_float4(v[u], v[u + 1], v[u + 2], v[u + 3]);
            }
          }
        }
      } else if (EPI == EPI_GATE) {
        // g = softmax(logits) over channels; m = 0 when the weight bound allows (no max
        // pass, see wimage_kernel), else the row max.
        float m = 0.f;
        if (!noshift) {
          m = -INFINITY;
#pragma unroll
          for (int c0 = 0; c0 < DH; c0 += 16) {
            uint32_t r[16];
            tc::tmem_ld16(acc + c0, r);
            tc::tmem_ld_wait();
#pragma unroll
            for (int u = 0; u < 16; ++u) m = fmaxf(m, __uint_as_float(r[u]) * un);
          }
          xg[hf * 128 + row] = m;
          group_bar(g);
          m = fmaxf(m, xg[(hf ^ 1) * 128 + row]);
        }
        const float unL = un * LOG2E, mL = m * LOG2E;
        float sum = 0.f;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) sum += ex2(fmaf(__uint_as_float(r[u]), unL, -mL));
        }
        xg[256 + hf * 128 + row] = sum;
        group_bar(g);
        sum = hf == 0 ? sum + xg[256 + 128 + row] : xg[256 + row] + sum;   // fixed order
        const float inv = fast_rcp(sum);
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = ex2(fmaf(__uint_as_float(r[u]), unL, -mL)) * inv;
          warp_store_chunk<D>(wbuf, a.out, wrow0, wrows, cb + c0, o, lane);
        }
      } else {
        float pp = 0.f, qq = 0.f;
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; u += 4) {
            if (EPI == EPI_NODE) {
              const float4 as4 = *reinterpret_cast<const float4 *>(s.avec + cb + c0 + u);
              const float4 ad4 = *reinterpret_cast<const float4 *>(s.avec + D + cb + c0 + u);
              const float asv[4] = {as4.x, as4.y, as4.z, as4.w};
              const float adv[4] = {ad4.x, ad4.y, ad4.z, ad4.w};
#pragma unroll
              for (int t = 0; t < 4; ++t) {
                o[u + t] = lrelu(__uint_as_float(r[u + t]) * un, a.slope);
                pp = fmaf(o[u + t], asv[t], pp);
                qq = fmaf(o[u + t], adv[t], qq);
              }
            } else {
              const float cexp = -aux * un * LOG2E;
#pragma unroll
              for (int t = 0; t < 4; ++t)                                      // e' (R2, R3)
                o[u + t] = fast_rcp(1.f + ex2(__uint_as_float(r[u + t]) * cexp));
            }
          }
          warp_store_chunk<D>(wbuf, a.out, wrow0, wrows, cb + c0, o, lane);
        }
        if (EPI == EPI_NODE) {
          xg[hf * 128 + row] = pp;
          xg[256 + hf * 128 + row] = qq;
          group_bar(g);
          if (hf == 0 && live) {
            a.p[grow] = pp + xg[128 + row];
            a.q[grow] = qq + xg[256 + 128 + row];
          }
        }
      }
      tc::fence_before_sync();
      tc::mbar_arrive(s.accfree + j);
      group_bar(g);        // the exchange buffer is reused by the next tile
    }
    TT_FLUSH(10 + wi);
  }
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  if (warp == 1) tc::tmem_dealloc<TMEM_COLS>(tmem);
#ifdef OCCU_TC_TIMING
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    g_tc_time[31][1] += clock64() - t_entry;
    g_tc_time[31][2] += 1;
  }
#endif
}

// ---------------------------------------------------------------------------
// d = 256, the paper's hidden width (P273 "hidden dimension of all the layers to 256"):
// the same three forward row-GEMMs (EPI_NODE / EPI_EDGE / EPI_GATE, same fused epilogues and
// fp16x2 split as rowgemm_kernel) on a CTA PAIR.  One CTA cannot hold the fp16x2 images of
// a 256 x 256 matrix (2 x 128 KB > 227 KB of shared memory), so two CTAs of a cluster on
// neighbouring SMs run tcgen05.mma.cta_group::2: M = 256 rows per MMA (128 per CTA), B split
// along N (each CTA keeps the images of its 128 output channels, resident for the whole
// kernel).  Each CTA ends up with full 256-channel rows in its TMEM, so the row epilogues
// (p/q dots, channel softmax) need no exchange between the CTAs.
//   warp 0      producer: the CTA's N-half of the images (bulk copies), then TMA boxes
//               (128 rows x 32 fp32, SW128) of its rows into a P_NS-box ring;
//   warp 1      TMEM (512 columns, cta_group::2 alloc in both CTAs); in the leader CTA the MMA
//               issuer: per 64-wide K chunk 4 x 3 tcgen05.mma.cta_group::2 (M=256, N=256,
//               K=16, A from TMEM, B from shared memory), each chunk committed to both CTAs'
//               A-slot-free barriers, each tile to both accumulator-full barriers;
//   warps 2-5   converters, thread = row: the row's 32 fp32 of a box -> the box slot is
//               released at once -> fp16x2 split -> tcgen05.st into a 4-chunk TMEM ring of A
//               operands (hi | lo); node inputs are scaled by 2^e_row from a per-row exponent
//               array (row_exp_kernel); one arrive per warp and chunk on the LEADER's A-full
//               barrier;
//   warps 6-21  epilogue, thread = (row, 64-channel quarter): its 64 accumulator values are
//               loaded (tcgen05.ld) and the accumulator released on the leader's barrier
//               before any arithmetic; the row epilogue (quarters combined in fixed order
//               through shared memory) then runs from registers, coalesced stores.
// TMEM per CTA: ACC [0, 256) + A ring [256, 512) (4 chunks x (32 hi + 32 lo columns)).  The
// shared-memory box ring is released as soon as a box is in registers, so the TMA stream runs
// up to a tile ahead of the MMAs (the resident images leave only ~64 KB for staging).  Pair
// tile t covers rows [256t, 256t + 256): rows [256t + 128·rank, +128) live in CTA `rank`.
// ---------------------------------------------------------------------------
constexpr int P_NTH = 704;           // warp 0 producer, 1 MMA, 2-5 converters, 6-21 epilogue
constexpr int P_EPI0 = 6;
constexpr int P_NS = 4;               // shared-memory ring of fp32 boxes (16 KB each)
constexpr int P_NA = 4;               // TMEM ring of A chunks (64 columns each)
#ifndef OCCU_PAIR_PF
#define OCCU_PAIR_PF 0
#endif
constexpr int P_PF = OCCU_PAIR_PF;    // boxes prefetched into L2 ahead of the shared-memory ring
constexpr int PD = 256;

struct PairSmem {
  uint8_t *w0, *w1;                   // this CTA's N-half of [w0 | w1]: [Kpad/64][128 rows][128 B]
  float *ring;                        // P_NS x 4096 floats
  uint64_t *full, *empty;             // [P_NS]
  uint64_t *afull, *afree;            // [P_NA]
  uint64_t *accfull, *accfree, *wfull, *wpeer;
  uint32_t *tmem_slot;
  float *avec;                        // [2][256] a_s, a_d (NODE)
  float *xch;                         // [2 values][4 quarters][128 rows]
  float *xbuf;                        // 16 epilogue warps x 16 x 20 floats
  uint64_t *eready;                   // [4] row exponents of tile i in erow (local row max)
  int *erow;                          // [4][128]
};

// nimg: 2 fp16x2 images (OCCU_FP32) or 1 BF16 image (OCCU_BF16)
__host__ __device__ inline size_t pair_smem_bytes(int K, int nimg) {
  const size_t img = size_t(kpad_of(K)) * 128 * 2;
  return 1024 + nimg * img + size_t(P_NS) * 16384 + 256 + 2048 + 4096 + 16 * 16 * 20 * 4 + 4 * 128 * 4;
}

__device__ __forceinline__ PairSmem carve_pair(uint8_t *raw, int K, int nimg) {
  PairSmem s;
  const uint32_t a = tc::smem_u32(raw);
  uint8_t *base = raw + ((1024 - (a & 1023)) & 1023);
  const size_t img = size_t(kpad_of(K)) * 128 * 2;
  s.w0 = base;
  s.w1 = base + img;
  s.ring = reinterpret_cast<float *>(base + nimg * img);
  uint8_t *misc = base + nimg * img + size_t(P_NS) * 16384;
  uint64_t *bars = reinterpret_cast<uint64_t *>(misc);
  s.full = bars;
  s.empty = bars + P_NS;
  s.afull = bars + 2 * P_NS;
  s.afree = s.afull + P_NA;
  s.accfull = s.afree + P_NA;
  s.accfree = s.accfull + 1;
  s.wfull = s.accfull + 2;
  s.wpeer = s.accfull + 3;
  s.eready = s.accfull + 4;           // 4
  s.tmem_slot = reinterpret_cast<uint32_t *>(misc + 224);
  s.avec = reinterpret_cast<float *>(misc + 256);
  s.xch = reinterpret_cast<float *>(misc + 256 + 2048);
  s.xbuf = reinterpret_cast<float *>(misc + 256 + 2048 + 4096);
  s.erow = reinterpret_cast<int *>(misc + 256 + 2048 + 4096 + 16 * 16 * 20 * 4);
  return s;
}

__device__ __forceinline__ void epi_bar_pair() { asm volatile("bar.sync 1, 512;" ::: "memory"); }

__device__ __forceinline__ uint32_t pack_bf16_rn(float x0, float x1) {
  const __nv_bfloat162 b = __floats2bfloat162_rn(x0, x1);
  return *reinterpret_cast<const uint32_t *>(&b);
}
// 16 channels of the thread's row: FP32 through the coalescing transpose; BF16 as one
// 32-byte sector per row
template <bool BF>
__device__ __forceinline__ void pair_store(float *wbuf, float *out, long wrow0, int wrows, long grow,
                                           bool live, int c0, const float (&o)[16], int lane) {
  if (BF) {
    if (!live) return;
    uint32_t w[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) w[u] = pack_bf16_rn(o[2 * u], o[2 * u + 1]);
    uint4 *dst = reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(out) + grow * PD + c0);
    dst[0] = make_uint4(w[0], w[1], w[2], w[3]);
    dst[1] = make_uint4(w[4], w[5], w[6], w[7]);
  } else {
    warp_store_chunk<PD>(wbuf, out, wrow0, wrows, c0, o, lane);
  }
}

// BF: OCCU_BF16 (one BF16 image, one product per K step, BF16 outputs, no row scale);
// AF32: the input rows are FP32 (every FP32-mode input; the layer-1 node features in BF16
// mode), else BF16 rows (TMA boxes of 128 rows x 64 bf16).
template <int EPI, bool BF, bool AF32>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(P_NTH, 1)
    rowgemm_pair_kernel(const __grid_constant__ CUtensorMap tmap, RowGemmArgs a) {
  extern __shared__ uint8_t smem_raw[];
  constexpr int EPB = AF32 ? 32 : 64;                          // K elements per box
  const int K = a.K, Kpad = kpad_of(K), NC = Kpad / 64, NB = (K + EPB - 1) / EPB;
  PairSmem s = carve_pair(smem_raw, K, BF ? 1 : 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = tc::cluster_rank();

  pdl_trigger();
  if (threadIdx.x == 0) {
    for (int j = 0; j < P_NS; ++j) {
      tc::mbar_init(s.full + j, 1);
      tc::mbar_init(s.empty + j, 128);  // the 4 converter warps
    }
    for (int j = 0; j < P_NA; ++j) {
      tc::mbar_init(s.afull + j, 8);    // 4 converter warps x 2 CTAs (leader's copy used)
      tc::mbar_init(s.afree + j, 1);    // multicast commit
    }
    tc::mbar_init(s.accfull, 1);        // multicast commit
    tc::mbar_init(s.accfree, 32);       // 16 epilogue warps x 2 CTAs (leader's copy used)
    tc::mbar_init(s.wfull, 1);
    tc::mbar_init(s.wpeer, 1);
    for (int j = 0; j < 4; ++j) tc::mbar_init(s.eready + j, 128);
    tc::fence_mbar_init();
  }
  if (warp == 1) tc::tmem_alloc2<TMEM_COLS>(s.tmem_slot);
  pdl_wait();
  const int fexp = __ldg(a.wfexp);
  const bool noshift = __ldg(a.wfexp + 1) != 0;
  if (EPI == EPI_NODE)
    for (int i = threadIdx.x; i < PD; i += P_NTH) {
      s.avec[i] = a.a_s[i];
      s.avec[PD + i] = a.a_d[i];
    }
  tc::fence_before_sync();
  __syncthreads();
  tc::cluster_sync();                 // both CTAs: barriers initialised, TMEM allocated
  tc::fence_after_sync();
  const uint32_t tmem = *s.tmem_slot;

  const int tiles = (a.R + 2 * TM - 1) / (2 * TM);
  const int cid = int(tc::cluster_id_x()), ncl = int(tc::ncluster_x());
  const int my = cid < tiles ? (tiles - 1 - cid) / ncl + 1 : 0;
  auto row0_of = [&](int i) -> long {
    int t = cid + i * ncl;
    if (a.rev) t = tiles - 1 - t;
    return long(t) * (2 * TM) + long(rank) * TM;
  };

  if (warp == 0) {
    // ---------------- producer ----------------
    if (lane == 0) {
      tc::prefetch_tmap(&tmap);
      const uint32_t ib = uint32_t(Kpad) * PD * 2;            // one full image (w0 or w1)
      tc::mbar_arrive_expect_tx(s.wfull, uint32_t(Kpad) * 128u * 2u * (BF ? 1u : 2u));
      for (int c = 0; c < NC; ++c) {                          // 16 KB per 64-wide K chunk
        const uint32_t src = uint32_t(c) * 32768u + rank * 16384u;
        tc::bulk_g2s(s.w0 + c * 16384, a.wimg + src, 16384, s.wfull);
        if (!BF) tc::bulk_g2s(s.w1 + c * 16384, a.wimg + ib + src, 16384, s.wfull);
      }
      if (rank == 1) {                                       // tell the leader its B half is in
        tc::mbar_wait(s.wfull, 0);
        tc::mbar_arrive_cluster(s.wpeer, 0);
      }
      // boxes are prefetched into L2 P_PF ahead of the ring: the resident weight images leave
      // room for only P_NS boxes in shared memory, too few bytes in flight to cover HBM latency
      const long nq = long(my) * NB;
      auto prefetch = [&](long qq) {
        if (qq >= nq) return;
        const long rr = row0_of(int(qq / NB));
        if (rr < a.R) tc::tma_prefetch_2d(&tmap, EPB * int(qq % NB), int(rr));
      };
      for (long qq = 0; qq < P_PF; ++qq) prefetch(qq);
      long q = 0;
      TT_DECL
      for (int i = 0; i < my; ++i) {
        const long r0 = row0_of(i);
        for (int b = 0; b < NB; ++b, ++q) {
          const int sl = int(q % P_NS);
          prefetch(q + P_PF);
          TT_WAIT_BEGIN
          if (q >= P_NS) tc::mbar_wait(s.empty + sl, uint32_t((q / P_NS) - 1) & 1u);
          TT_WAIT_END
          if (r0 < a.R) {
            tc::mbar_arrive_expect_tx(s.full + sl, 16384u);
            tc::tma_load_2d(s.ring + sl * 4096, &tmap, EPB * b, int(r0), s.full + sl);
          } else {
            tc::mbar_arrive(s.full + sl);                     // rows past R: nothing to load
          }
        }
      }
      if (EPI == EPI_GATE) TT_FLUSH(0);
    }
    __syncwarp();
  } else if (warp == 1) {
    // ---------------- MMA issuer (leader CTA) ----------------
    if (rank == 0) {
      const uint32_t idsc = tc::idesc(256, uint32_t(PD), BF ? tc::FMT_BF16 : tc::FMT_F16);
      const uint32_t w0a = tc::smem_u32(s.w0), w1a = tc::smem_u32(s.w1);
      const int nk = (K + 15) / 16;
      tc::mbar_wait(s.wfull, 0);
      tc::mbar_wait_cluster(s.wpeer, 0);
      TT_DECL
      for (int i = 0; i < my; ++i) {
        TT_WAIT_BEGIN
        if (i >= 1) tc::mbar_wait_cluster(s.accfree, uint32_t(i - 1) & 1u);
        TT_WAIT_END
        for (int c = 0; c < NC; ++c) {
          const long qa = long(i) * NC + c;
          const int as = int(qa % P_NA);
          TT_WAIT_BEGIN
          tc::mbar_wait_cluster(s.afull + as, uint32_t(qa / P_NA) & 1u);
          TT_WAIT_END
          tc::fence_after_sync();
          if (lane == 0) {
            const uint32_t ah = tmem + 256u + uint32_t(as) * 64u;
            for (int kk = 0; kk < 4 && 4 * c + kk < nk; ++kk) {
              const uint32_t bo = uint32_t(c) * 16384u + uint32_t(kk) * 32u;
              const uint64_t b0 = tc::sdesc_sw128(w0a + bo), b1 = tc::sdesc_sw128(w1a + bo);
              const uint32_t a0 = ah + uint32_t(kk) * 8u, a1 = a0 + 32u;
              tc::mma2_f16_ts(tmem, a0, b0, idsc, (c | kk) ? 1u : 0u);
              if (!BF) {
                tc::mma2_f16_ts(tmem, a0, b1, idsc, 1u);
                tc::mma2_f16_ts(tmem, a1, b0, idsc, 1u);
              }
            }
            tc::mma2_commit_both(s.afree + as);
            if (c == NC - 1) tc::mma2_commit_both(s.accfull);
          }
          __syncwarp();
        }
      }
      if (EPI == EPI_GATE) TT_FLUSH(1);
    }
  } else if (warp < P_EPI0) {
    // ---------------- converters: thread = row -> TMEM A ring ----------------
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    TT_DECL
    for (int i = 0; i < my; ++i) {
      const long r0 = row0_of(i);
      const bool live = long(row) < a.R - r0;
      float xs = 1.f;                                          // e' in [0, 1]: unscaled
      if (!BF && EPI == EPI_NODE) {
        if (a.rexp) {                                          // exponents from row_exp_kernel
          if (live) xs = ldexpf(1.f, __ldg(a.rexp + r0 + row));
        } else {
          // K <= 128: the tile's NB <= P_NS boxes are all in the ring at once; the row max
          // is taken over them before any box is released (no row_exp_kernel pass)
          float mx = 0.f;
          for (int b = 0; b < NB; ++b) {
            const long q = long(i) * NB + b;
            const int sl = int(q % P_NS);
            tc::mbar_wait(s.full + sl, uint32_t(q / P_NS) & 1u);
            const float *box = s.ring + sl * 4096;
            if (live)
#pragma unroll
              for (int u = 0; u < 8; ++u)
                if (32 * b + 4 * u < K) {
                  const float4 v = slot_ld4(box, row, 4 * u);
                  mx = fmaxf(mx, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w))));
                }
          }
          const int er = scale_exp(mx);
          xs = ldexpf(1.f, er);
          s.erow[(i & 3) * 128 + row] = er;
          tc::mbar_arrive(s.eready + (i & 3));
        }
      }
      for (int c = 0; c < NC; ++c) {
        const long qa = long(i) * NC + c;
        const int as = int(qa % P_NA);
        if (!AF32) {
          // BF16 rows: one box per chunk, the row's 128 B copied into the TMEM ring as is
          const long q = long(i) * NB + c;
          const int sl = int(q % P_NS);
          tc::mbar_wait(s.full + sl, uint32_t(q / P_NS) & 1u);
          const uint8_t *box = reinterpret_cast<const uint8_t *>(s.ring + sl * 4096);
          uint32_t w[32];
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            uint4 x = make_uint4(0u, 0u, 0u, 0u);
            if (live && 64 * c + 8 * u < K)
              x = *reinterpret_cast<const uint4 *>(box + row * 128 + ((u ^ (row & 7)) << 4));
            w[4 * u] = x.x; w[4 * u + 1] = x.y; w[4 * u + 2] = x.z; w[4 * u + 3] = x.w;
          }
          tc::mbar_arrive(s.empty + sl);
          if (qa >= P_NA) tc::mbar_wait(s.afree + as, uint32_t((qa / P_NA) - 1) & 1u);
          tc::tmem_st32(lane_base + 256u + uint32_t(as) * 64u, w);
          tc::tmem_st_wait();
          tc::fence_before_sync();
          __syncwarp();
          if (lane == 0) tc::mbar_arrive_cluster(s.afull + as, 0);
          continue;
        }
        for (int kh = 0; kh < 2; ++kh) {
          const int b = 2 * c + kh;
          if (b >= NB) break;
          const long q = long(i) * NB + b;
          const int sl = int(q % P_NS);
          TT_WAIT_BEGIN
          tc::mbar_wait(s.full + sl, uint32_t(q / P_NS) & 1u);
          TT_WAIT_END
          const float *box = s.ring + sl * 4096;
          float4 v[8];
#pragma unroll
          for (int u = 0; u < 8; ++u)
            v[u] = (live && 32 * b + 4 * u < K) ? slot_ld4(box, row, 4 * u) : make_float4(0.f, 0.f, 0.f, 0.f);
          tc::mbar_arrive(s.empty + sl);                      // the box is in registers
          uint32_t h[16], l[16];
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            float4 x = v[u];
            if (!BF && EPI == EPI_NODE) {
              x.x *= xs; x.y *= xs; x.z *= xs; x.w *= xs;
            }
            if (BF) {                                          // FP32 rows rounded to BF16 (RN)
              h[2 * u] = pack_bf16_rn(x.x, x.y);
              h[2 * u + 1] = pack_bf16_rn(x.z, x.w);
            } else {
              split2(x.x, x.y, h[2 * u], l[2 * u]);
              split2(x.z, x.w, h[2 * u + 1], l[2 * u + 1]);
            }
          }
          TT_WAIT_BEGIN
          if (kh == 0 && qa >= P_NA) tc::mbar_wait(s.afree + as, uint32_t((qa / P_NA) - 1) & 1u);
          TT_WAIT_END
          const uint32_t col = 256u + uint32_t(as) * 64u + uint32_t(kh) * 16u;
          tc::tmem_st16(lane_base + col, h);
          if (!BF) tc::tmem_st16(lane_base + col + 32u, l);
        }
        tc::tmem_st_wait();
        tc::fence_before_sync();
        __syncwarp();
        if (lane == 0) tc::mbar_arrive_cluster(s.afull + as, 0);
      }
    }
    if (EPI == EPI_GATE) TT_FLUSH(2 + (warp - 2));
    // the last chunks' MMAs (and their commits to this CTA) must land before teardown
    for (long qa = max(0L, long(my) * NC - P_NA); qa < long(my) * NC; ++qa)
      tc::mbar_wait(s.afree + int(qa % P_NA), uint32_t(qa / P_NA) & 1u);
  } else {
    // ---------------- epilogue: thread = (row, 64-channel quarter) ----------------
    // the thread's 64 accumulator values are loaded at once and the accumulator released
    // before any arithmetic, so the next tile's MMAs overlap this tile's epilogue
    const int wi = warp - P_EPI0;
    const int cq = wi >> 2;
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    float *wbuf = s.xbuf + wi * (16 * 20);
    constexpr int DQ = PD / 4;
    const int cb = cq * DQ;
    TT_DECL
    for (int i = 0; i < my; ++i) {
      const long r0 = row0_of(i);
      const int nrows = int(max(0L, min(long(TM), a.R - r0)));
      const bool live = row < nrows;
      float aux = 0.f;
      if (EPI == EPI_EDGE && live)
        aux = __ldg(a.pin + __ldg(a.src + r0 + row)) + __ldg(a.qin + __ldg(a.dst + r0 + row));  // α
      int er = 0;
      if (!BF && EPI == EPI_NODE) {
        if (a.rexp) {
          if (live) er = __ldg(a.rexp + r0 + row);
        } else {
          tc::mbar_wait(s.eready + (i & 3), uint32_t(i >> 2) & 1u);
          er = s.erow[(i & 3) * 128 + row];
        }
      }
      TT_WAIT_BEGIN
      tc::mbar_wait(s.accfull, uint32_t(i) & 1u);
      TT_WAIT_END
      tc::fence_after_sync();
      uint32_t r[DQ];
      {
        uint32_t (&r0_)[16] = *reinterpret_cast<uint32_t (*)[16]>(r);
        uint32_t (&r1_)[16] = *reinterpret_cast<uint32_t (*)[16]>(r + 16);
        uint32_t (&r2_)[16] = *reinterpret_cast<uint32_t (*)[16]>(r + 32);
        uint32_t (&r3_)[16] = *reinterpret_cast<uint32_t (*)[16]>(r + 48);
        tc::tmem_ld16(lane_base + uint32_t(cb), r0_);
        tc::tmem_ld16(lane_base + uint32_t(cb) + 16u, r1_);
        tc::tmem_ld16(lane_base + uint32_t(cb) + 32u, r2_);
        tc::tmem_ld16(lane_base + uint32_t(cb) + 48u, r3_);
        tc::tmem_ld_wait();
      }
      tc::fence_before_sync();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive_cluster(s.accfree, 0);    // accumulator free
      const float un = ldexpf(1.f, -(er + fexp));
      const long grow = r0 + row;
      const long wrow0 = r0 + qd * 32;
      const int wrows = max(0, min(32, nrows - qd * 32));
      if (EPI == EPI_GATE) {
        float m = 0.f;
        if (!noshift) {
          m = -INFINITY;
#pragma unroll
          for (int u = 0; u < DQ; ++u) m = fmaxf(m, __uint_as_float(r[u]) * un);
          s.xch[cq * 128 + row] = m;
          epi_bar_pair();
          m = fmaxf(fmaxf(s.xch[row], s.xch[128 + row]), fmaxf(s.xch[256 + row], s.xch[384 + row]));
        }
        const float unL = un * LOG2E, mL = m * LOG2E;
        float sum = 0.f;
#pragma unroll
        for (int u = 0; u < DQ; ++u) {
          const float e = ex2(fmaf(__uint_as_float(r[u]), unL, -mL));
          r[u] = __float_as_uint(e);
          sum += e;
        }
        float *xs2 = s.xch + 512;
        xs2[cq * 128 + row] = sum;
        epi_bar_pair();
        sum = ((xs2[row] + xs2[128 + row]) + xs2[256 + row]) + xs2[384 + row];   // fixed order
        const float inv = fast_rcp(sum);
#pragma unroll
        for (int u = 0; u < DQ; ++u) r[u] = __float_as_uint(__uint_as_float(r[u]) * inv);
#pragma unroll
        for (int c0 = 0; c0 < DQ; c0 += 16)
          pair_store<BF>(wbuf, a.out, wrow0, wrows, grow, live, cb + c0,
                         *reinterpret_cast<const float (*)[16]>(r + c0), lane);
      } else {
        float pp = 0.f, qq = 0.f;
#pragma unroll
        for (int c0 = 0; c0 < DQ; c0 += 16) {
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; u += 4) {
            if (EPI == EPI_NODE) {
              const float4 as4 = *reinterpret_cast<const float4 *>(s.avec + cb + c0 + u);
              const float4 ad4 = *reinterpret_cast<const float4 *>(s.avec + PD + cb + c0 + u);
              const float asv[4] = {as4.x, as4.y, as4.z, as4.w};
              const float adv[4] = {ad4.x, ad4.y, ad4.z, ad4.w};
#pragma unroll
              for (int t = 0; t < 4; ++t) {
                o[u + t] = lrelu(__uint_as_float(r[c0 + u + t]) * un, a.slope);
                pp = fmaf(o[u + t], asv[t], pp);
                qq = fmaf(o[u + t], adv[t], qq);
              }
            } else {
              const float cexp = -aux * un * LOG2E;
#pragma unroll
              for (int t = 0; t < 4; ++t) o[u + t] = fast_rcp(1.f + ex2(__uint_as_float(r[c0 + u + t]) * cexp));
            }
          }
          pair_store<BF>(wbuf, a.out, wrow0, wrows, grow, live, cb + c0, o, lane);
        }
        if (EPI == EPI_NODE) {
          s.xch[cq * 128 + row] = pp;
          s.xch[512 + cq * 128 + row] = qq;
          epi_bar_pair();
          if (cq == 0 && live) {
            a.p[grow] = ((s.xch[row] + s.xch[128 + row]) + s.xch[256 + row]) + s.xch[384 + row];
            a.q[grow] = ((s.xch[512 + row] + s.xch[640 + row]) + s.xch[768 + row]) + s.xch[896 + row];
          }
        }
      }
      epi_bar_pair();          // the exchange area is reused by the next tile
    }
    if (EPI == EPI_GATE) TT_FLUSH(6 + wi);
  }
  tc::fence_before_sync();
  __syncthreads();
  tc::cluster_sync();
  tc::fence_after_sync();
  if (warp == 1) tc::tmem_dealloc2<TMEM_COLS>(tmem);
}

// Per-row power-of-two scale exponent e_r (max|x_r|·2^e_r in [2^14, 2^15), scale_exp) of the
// node-transform input rows at d = 256; warp per row.
__global__ void __launch_bounds__(256) row_exp_kernel(const float *__restrict__ A, int R, int K,
                                                      int *__restrict__ out) {
  pdl_trigger();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  for (long r = (long(blockIdx.x) * 256 + threadIdx.x) / 32; r < R; r += long(gridDim.x) * 8) {
    float mx = 0.f;
    for (int k = 4 * lane; k < K; k += 128) {
      const float4 v = __ldg(reinterpret_cast<const float4 *>(A + r * K + k));
      mx = fmaxf(mx, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w))));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if (lane == 0) out[r] = scale_exp(mx);
  }
}

// ---------------------------------------------------------------------------
// Fused edge transform + channel-softmax gate of one ANEE layer (a3 + a4, P145/P149):
//   e' = σ(α · W_e e_in), α = p[s] + q[t];   g = softmax_c(W_m e')
// e' is written once (next layer's input, kept for the backward) and never re-read
// by the gate.  Persistent, one CTA per SM, 128-edge tiles, two chained tcgen05
// GEMMs per tile (fp16x2-split operands, 3 products, FP32 accumulation in TMEM):
//   warp 0       producer: TMA boxes (128 rows x 32 fp32) of e_in into a per-box ring
//   warp 1       MMA: ACC1 = A1·W_eᵀ, ACC2 = A2·W_mᵀ (A from TMEM, B = weight images)
//   warps 2-9    converters: e_in (in (0,1), unscaled) -> fp16x2 -> TMEM A1
//   warps 10-17  stage 1: z = ACC1·2^-f_e, e' = σ(αz) -> HBM and fp16x2 -> TMEM A2
//   warps 18-25  stage 2: softmax(ACC2·2^-f_m) -> HBM g
// FIRST (layer 1, F_e <= 16): no A1 / MMA1; stage 1 forms z = W_e e0 on CUDA cores from
// the raw edge_feat rows gathered through in_eid (a1 fused), writing e0_out if asked.
// TMEM columns: A1 [0,128) ACC1 [128,256) A2 [256,384) ACC2 [384,512), single-buffered;
// the MMA warp issues MMA1(i) before MMA2(i-1) so stage 1 never waits on stage 2.
// ---------------------------------------------------------------------------
struct EdgeGateArgs {
  const float *e_in; int Ke, R;      // [R][Ke] (FIRST: raw edge_feat [R][Ke], row eid[k])
  const int32_t *eid;                // FIRST: in-CSR edge -> edge_feat row
  const float *W_e;                  // FIRST: [D][Ke] fp32 (CUDA-core path)
  const uint8_t *wimg_e, *wimg_m;    // fp16x2 images [w0 | w1]
  const int *wf_e, *wf_m;            // scale exponents (wf_m[1] = softmax no-shift flag)
  const float *p, *q;
  const int32_t *src, *dst;
  float *e_out, *e0_out, *g;        // e_out nullable (last inference layer: e' is not needed)
  int rev;
  int dbg;                           // sensitivity experiments only (OCCU_EG_DBG), 0 in production
  // AGG (a4 + a5 + a6 fused into stage 2, inference): m = g ⊙ h̄[s] summed over each
  // destination's dst-sorted in-edges inside the warp's 32 rows; complete segments -> h_out
  // (LReLU, ÷ deg for MEAN), segments crossing a 32-edge unit -> part (agg_fixup_kernel)
  const float *hbar;
  const int32_t *in_ptr;
  float *h_out, *part;
  int mean;
  float slope;
};

constexpr int EG_NTH = 832;

__host__ __device__ inline size_t eg_smem_bytes(int D, int Ke, bool first) {
  const size_t imgm = size_t(D) * D * 2;
  const size_t imge = first ? size_t(Ke) * D * 4 / 2 : size_t(kpad_of(Ke)) * D * 2;  // 2 x imge total
  const size_t ring = first ? 0 : size_t(nbox_of(Ke)) * 16384;
  return 1024 + 2 * imgm + 2 * imge + ring + 256 + 2 * 2 * 128 * 4 + 16 * 16 * 20 * 4;
}

template <int D, int KM, bool AGG = false>   // KM > 0: FIRST (layer-1 CUDA-core edge transform, Ke <= KM)
__global__ void __launch_bounds__(EG_NTH, 1) edgegate_kernel(const __grid_constant__ CUtensorMap tmap,
                                                             EdgeGateArgs a) {
  constexpr bool FIRST = KM > 0;
  constexpr int KMX = FIRST ? KM : 1;
  extern __shared__ uint8_t smem_raw[];
  const int Ke = a.Ke, NB = FIRST ? 0 : nbox_of(Ke), Kpe = FIRST ? Ke : kpad_of(Ke);
  uint8_t *base = smem_raw + ((1024 - (tc::smem_u32(smem_raw) & 1023)) & 1023);
  const size_t imgm = size_t(D) * D * 2;
  const size_t imge = FIRST ? size_t(Ke) * D * 4 / 2 : size_t(Kpe) * D * 2;
  uint8_t *wm0 = base, *wm1 = base + imgm, *we0 = base + 2 * imgm, *we1 = we0 + imge;
  float *ring = reinterpret_cast<float *>(we0 + 2 * imge);
  uint8_t *misc = reinterpret_cast<uint8_t *>(ring) + (FIRST ? 0 : size_t(NB) * 16384);
  uint64_t *bars = reinterpret_cast<uint64_t *>(misc);
  uint64_t *full = bars, *empty = bars + 4, *a1full = bars + 8, *a1free = bars + 9,
           *acc1full = bars + 10, *acc1free = bars + 11, *a2full = bars + 12, *a2free = bars + 13,
           *acc2full = bars + 14, *acc2free = bars + 15, *wfull = bars + 16;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(misc + 160);
  float *xg = reinterpret_cast<float *>(misc + 256);                 // stage 2: [2][2][128]
  float *xbuf = xg + 2 * 2 * 128;                                    // 16 warps x 16 x 20
  float *wt = reinterpret_cast<float *>(we0);                        // FIRST: W_eᵀ [Ke][D]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (FIRST)
    for (int i = threadIdx.x; i < D * Ke; i += EG_NTH) wt[(i % Ke) * D + i / Ke] = a.W_e[i];
  if (threadIdx.x == 0) {
    for (int j = 0; j < 4; ++j) {
      tc::mbar_init(full + j, 1);
      tc::mbar_init(empty + j, 128);
    }
    tc::mbar_init(a1full, 256);
    tc::mbar_init(a1free, 1);
    tc::mbar_init(acc1full, 1);
    tc::mbar_init(acc1free, 256);
    tc::mbar_init(a2full, 256);
    tc::mbar_init(a2free, 1);
    tc::mbar_init(acc2full, 1);
    tc::mbar_init(acc2free, 256);
    tc::mbar_init(wfull, 1);
    tc::fence_mbar_init();
  }
  if (warp == 1) tc::tmem_alloc<TMEM_COLS>(tmem_slot);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  const uint32_t tmem = *tmem_slot;
  constexpr uint32_t A1 = 0, ACC1 = 128, A2 = 256, ACC2 = 384;
  const int tiles = (a.R + TM - 1) / TM;
  const int my = blockIdx.x < tiles ? (tiles - 1 - int(blockIdx.x)) / int(gridDim.x) + 1 : 0;
  auto tile_r0 = [&](int i) -> long {
    const int t = int(blockIdx.x) + i * int(gridDim.x);
    return long(a.rev ? tiles - 1 - t : t) * TM;
  };

  if (warp == 0) {
    if (lane == 0) {
      if (!FIRST) tc::prefetch_tmap(&tmap);
      const uint32_t bm = uint32_t(imgm), be = FIRST ? 0u : uint32_t(imge);
      tc::mbar_arrive_expect_tx(wfull, 2 * bm + 2 * be);
      for (uint32_t o = 0; o < bm; o += 16384) {
        const uint32_t n = bm - o < 16384 ? bm - o : 16384;
        tc::bulk_g2s(wm0 + o, a.wimg_m + o, n, wfull);
        tc::bulk_g2s(wm1 + o, a.wimg_m + bm + o, n, wfull);
      }
      for (uint32_t o = 0; o < be; o += 16384) {
        const uint32_t n = be - o < 16384 ? be - o : 16384;
        tc::bulk_g2s(we0 + o, a.wimg_e + o, n, wfull);
        tc::bulk_g2s(we1 + o, a.wimg_e + be + o, n, wfull);
      }
      TT_DECL
      if (!FIRST)
        for (int i = 0; i < my; ++i) {
          const int r0 = int(tile_r0(i));
          for (int b = 0; b < NB; ++b) {
            TT_WAIT_BEGIN
            if (i >= 1) tc::mbar_wait(empty + b, (i - 1) & 1);
            TT_WAIT_END
            tc::mbar_arrive_expect_tx(full + b, 16384u);
            tc::tma_load_2d(ring + b * 4096, &tmap, 32 * b, r0, full + b);
          }
        }
      TT_FLUSH_EG(0);
    }
    __syncwarp();
  } else if (warp == 1) {
    const uint32_t idsc = tc::idesc(128, uint32_t(D), tc::FMT_F16);
    const uint32_t m0 = tc::smem_u32(wm0), m1 = tc::smem_u32(wm1);
    const uint32_t e0a = tc::smem_u32(we0), e1a = tc::smem_u32(we1);
    tc::mbar_wait(wfull, 0);
    auto gemm = [&](uint32_t acc, uint32_t aop, uint32_t w0, uint32_t w1, int K, int Kp) {
      for (int kk = 0; kk < K / 16; ++kk) {
        const uint32_t boff = uint32_t(kk >> 2) * uint32_t(D) * 128u + uint32_t(kk & 3) * 32u;
        const uint64_t b0 = tc::sdesc_sw128(w0 + boff), b1 = tc::sdesc_sw128(w1 + boff);
        const uint32_t x0 = tmem + aop + uint32_t(kk) * 8u, x1 = x0 + uint32_t(Kp / 2);
        tc::mma_f16_ts(tmem + acc, x0, b0, idsc, kk > 0 ? 1u : 0u);
        tc::mma_f16_ts(tmem + acc, x0, b1, idsc, 1u);
        tc::mma_f16_ts(tmem + acc, x1, b0, idsc, 1u);
      }
    };
    TT_DECL
    for (int i = 0; i <= my; ++i) {
      if (!FIRST && i < my) {                    // MMA1(i)
        TT_WAIT_BEGIN
        tc::mbar_wait(a1full, i & 1);
        if (i >= 1) tc::mbar_wait(acc1free, (i - 1) & 1);
        TT_WAIT_END
        tc::fence_after_sync();
        if (lane == 0) {
          gemm(ACC1, A1, e0a, e1a, Ke, Kpe);
          tc::mma_commit(acc1full);
          tc::mma_commit(a1free);
        }
        __syncwarp();
      }
      if (i >= 1) {                              // MMA2(i-1)
        const int t = i - 1;
        TT_WAIT_BEGIN
        tc::mbar_wait(a2full, t & 1);
        if (t >= 1) tc::mbar_wait(acc2free, (t - 1) & 1);
        TT_WAIT_END
        tc::fence_after_sync();
        if (lane == 0) {
          gemm(ACC2, A2, m0, m1, D, D);
          tc::mma_commit(acc2full);
          tc::mma_commit(a2free);
        }
        __syncwarp();
      }
    }
    TT_FLUSH_EG(1);
  } else if (warp < EPI0) {
    if (!FIRST) {
      // converters: thread = (row, K-half); e_in in (0,1) -> unscaled fp16x2 split
      const int qd = warp & 3, kh = (warp - 2) >> 2, row = qd * 32 + lane;
      const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
      const int KH = Kpe / 2, kb = kh * KH, bpb = NB / 2;   // boxes per half
      TT_DECL
      for (int i = 0; i < my; ++i) {
        const long r0 = tile_r0(i);
        const bool live = row < min(TM, int(a.R - r0));
        TT_WAIT_BEGIN
        for (int b = 0; b < bpb; ++b) tc::mbar_wait(full + kh * bpb + b, i & 1);
        if (i >= 1) tc::mbar_wait(a1free, (i - 1) & 1);
        TT_WAIT_END
        for (int c0 = 0; c0 < KH / 2; c0 += 16) {
          uint32_t x0[16], x1[16];
#pragma unroll
          for (int u = 0; u < 16; u += 2) {
            const int k = kb + 2 * (c0 + u);
            float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
            if (live && k < Ke) v = slot_ld4(ring, row, k);
            split2(v.x, v.y, x0[u], x1[u]);
            split2(v.z, v.w, x0[u + 1], x1[u + 1]);
          }
          const uint32_t col = A1 + uint32_t(kb / 2 + c0);
          tc::tmem_st16(lane_base + col, x0);
          tc::tmem_st16(lane_base + col + Kpe / 2, x1);
        }
        tc::tmem_st_wait();
        tc::fence_before_sync();
        for (int b = 0; b < bpb; ++b) tc::mbar_arrive(empty + kh * bpb + b);
        tc::mbar_arrive(a1full);
      }
      TT_FLUSH_EG(2 + (warp - 2));
    }
  } else if (warp < EPI0 + 8) {
    // ---- stage 1: e' = σ(α z) -> HBM + fp16x2 -> A2 (thread = row, half hf of D) ----
    const int wi = warp - EPI0, hf = wi >> 2, qd = warp & 3, row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    float *wbuf = xbuf + wi * (16 * 20);
    constexpr int DH = D / 2;
    const int cb = hf * DH;
    const float un = FIRST ? 1.f : ldexpf(1.f, -__ldg(a.wf_e));
    // software-pipelined row inputs: indices of tile i+2 and values of tile i+1 are in
    // flight while tile i is processed (α = p[s] + q[t] is a two-level gather)
    auto rows_of = [&](int i, long &grow) {
      const long r0 = tile_r0(i);
      grow = r0 + row;
      return i < my && row < min(TM, int(a.R - r0));
    };
    int s_n = 0, t_n = 0, x_n = 0;                   // indices of tile i+1
    auto load_idx = [&](int i, int &sv, int &tv, int &xv) {
      long gr;
      if (rows_of(i, gr)) {
        sv = __ldg(a.src + gr);
        tv = __ldg(a.dst + gr);
        if (FIRST) xv = a.eid ? __ldg(a.eid + gr) : int(gr);
      }
    };
    float al_n = 0.f, ev_n[KMX];
    auto load_val = [&](int i, int sv, int tv, int xv) {
      long gr;
      const bool lv = rows_of(i, gr);
      al_n = lv ? __ldg(a.p + sv) + __ldg(a.q + tv) : 0.f;                     // α (R1)
#pragma unroll
      for (int j = 0; j < KMX; ++j)
        ev_n[j] = (FIRST && lv && j < Ke) ? __ldg(a.e_in + long(xv) * Ke + j) : 0.f;
    };
    {
      int s0 = 0, t0 = 0, x0 = 0;
      load_idx(0, s0, t0, x0);
      load_val(0, s0, t0, x0);
      load_idx(1, s_n, t_n, x_n);
    }
    TT_DECL
    for (int i = 0; i < my; ++i) {
      const long r0 = tile_r0(i);
      const int nrows = min(TM, int(a.R - r0));
      const bool live = row < nrows;
      const long grow = r0 + row;
      const float al = al_n;
      float ev[KMX];
#pragma unroll
      for (int j = 0; j < KMX; ++j) ev[j] = ev_n[j];
      load_val(i + 1, s_n, t_n, x_n);                // tile i+1 values (indices ready)
      load_idx(i + 2, s_n, t_n, x_n);                // tile i+2 indices
      if (FIRST && a.e0_out && hf == 0 && live) {
#pragma unroll
        for (int j = 0; j < KMX; ++j)
          if (j < Ke) a.e0_out[grow * Ke + j] = ev[j];
      }
      TT_WAIT_BEGIN
      if (!FIRST) tc::mbar_wait(acc1full, i & 1);
      if (i >= 1) tc::mbar_wait(a2free, (i - 1) & 1);
      TT_WAIT_END
      tc::fence_after_sync();
      const float cexp = -al * un * LOG2E;
      const long wrow0 = r0 + qd * 32;
      const int wrows = max(0, min(32, nrows - qd * 32));
#pragma unroll 1
      for (int c0 = 0; c0 < DH; c0 += 16) {
        float z[16];
        if (FIRST) {
#pragma unroll
          for (int u = 0; u < 16; ++u) z[u] = 0.f;
#pragma unroll
          for (int j = 0; j < KMX; ++j) {
            if (j >= Ke) break;
            const float x = ev[j];
#pragma unroll
            for (int u = 0; u < 16; u += 4) {
              const float4 w = *reinterpret_cast<const float4 *>(wt + j * D + cb + c0 + u);
              z[u] = fmaf(w.x, x, z[u]); z[u + 1] = fmaf(w.y, x, z[u + 1]);
              z[u + 2] = fmaf(w.z, x, z[u + 2]); z[u + 3] = fmaf(w.w, x, z[u + 3]);
            }
          }
        } else {
          uint32_t r[16];
          tc::tmem_ld16(lane_base + ACC1 + cb + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) z[u] = __uint_as_float(r[u]);
        }
        float o[16];
        if (a.dbg & 1) {
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = fmaf(z[u], cexp, 0.5f);
        } else {
#pragma unroll
          for (int u = 0; u < 16; ++u)                                        // e' (R2, R3)
            o[u] = FIRST ? fast_rcp(1.f + fast_exp(-(al * z[u])))
                         : fast_rcp(1.f + ex2(z[u] * cexp));
        }
        uint32_t x0[8], x1[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) split2(o[2 * u], o[2 * u + 1], x0[u], x1[u]);
        const uint32_t col = A2 + uint32_t((cb + c0) / 2);
        tc::tmem_st8(lane_base + col, x0);
        tc::tmem_st8(lane_base + col + D / 2, x1);
        if (!(a.dbg & 4) && a.e_out) warp_store_chunk<D>(wbuf, a.e_out, wrow0, wrows, cb + c0, o, lane);
      }
      tc::tmem_st_wait();
      tc::fence_before_sync();
      if (!FIRST) tc::mbar_arrive(acc1free);
      tc::mbar_arrive(a2full);
    }
    TT_FLUSH_EG(10 + wi);
  } else {
    // ---- stage 2: g = softmax(ACC2 · 2^-f_m) -> HBM ----
    const int wi = warp - EPI0 - 8, hf = wi >> 2, qd = warp & 3, row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    float *wbuf = xbuf + (8 + wi) * (16 * 20);
    constexpr int DH = D / 2;
    const int cb = hf * DH;
    const float un = ldexpf(1.f, -__ldg(a.wf_m));
    const bool noshift = __ldg(a.wf_m + 1) != 0;
    TT_DECL
    for (int i = 0; i < my; ++i) {
      const long r0 = tile_r0(i);
      const int nrows = min(TM, int(a.R - r0));
      const long wrow0 = r0 + qd * 32;
      const int wrows = max(0, min(32, nrows - qd * 32));
      TT_WAIT_BEGIN
      tc::mbar_wait(acc2full, i & 1);
      TT_WAIT_END
      tc::fence_after_sync();
      const uint32_t acc = lane_base + ACC2 + cb;
      float m = 0.f;
      if (!noshift) {
        m = -INFINITY;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) m = fmaxf(m, __uint_as_float(r[u]) * un);
        }
        xg[hf * 128 + row] = m;
        group_bar(1);
        m = fmaxf(m, xg[(hf ^ 1) * 128 + row]);
      }
      const float unL = un * LOG2E, mL = m * LOG2E;
      float sum = 0.f;
#pragma unroll
      for (int c0 = 0; c0 < DH; c0 += 16) {
        uint32_t r[16];
        tc::tmem_ld16(acc + c0, r);
        tc::tmem_ld_wait();
#pragma unroll
        for (int u = 0; u < 16; ++u) sum += ex2(fmaf(__uint_as_float(r[u]), unL, -mL));
      }
      xg[256 + hf * 128 + row] = sum;
      group_bar(1);
      sum = hf == 0 ? sum + xg[256 + 128 + row] : xg[256 + row] + sum;   // fixed order
      const float inv = fast_rcp(sum);
      if constexpr (AGG) {
        // destination segments inside this warp's 32 consecutive (dst-sorted) edges
        const long grow = r0 + row;
        const bool live = row < nrows;
        const int tn = live ? __ldg(a.dst + grow) : -1 - lane;         // pad rows: own segment
        const int sn = live ? __ldg(a.src + grow) : 0;
        const int tprev = __shfl_up_sync(0xffffffffu, tn, 1);
        const int tnext = __shfl_down_sync(0xffffffffu, tn, 1);
        const bool head = lane == 0 || tprev != tn;
        const bool tail = lane == 31 || tnext != tn;
        const unsigned heads = __ballot_sync(0xffffffffu, head);
        const int start = 31 - __clz(heads & (0xffffffffu >> (31 - lane)));
        const int maxlen = __reduce_max_sync(0xffffffffu, unsigned(lane - start + 1));
        int beg = 0, end = 0;
        if (tail && live) {
          beg = __ldg(a.in_ptr + tn);
          end = __ldg(a.in_ptr + tn + 1);
        }
        const bool before = live && beg < wrow0 + start;               // segment began earlier
        const bool after = live && end > wrow0 + lane + 1;               // continues after this warp
        const float dsc = a.mean ? float(end - beg > 0 ? end - beg : 1) : 1.f;
        const float *hbr = a.hbar + long(sn) * D + cb;
        const long unit = wrow0 >> 5;
        float4 hpre[4];                                                  // h̄[s] one chunk ahead
#pragma unroll
        for (int u = 0; u < 4; ++u)
          hpre[u] = live ? __ldg(reinterpret_cast<const float4 *>(hbr) + u) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          float4 hc[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) hc[u] = hpre[u];
          if (c0 + 16 < DH)
#pragma unroll
            for (int u = 0; u < 4; ++u)
              hpre[u] = live ? __ldg(reinterpret_cast<const float4 *>(hbr + c0 + 16) + u) : make_float4(0.f, 0.f, 0.f, 0.f);
          tc::tmem_ld_wait();
          float v[16];
#pragma unroll
          for (int u = 0; u < 16; u += 4) {
            const float bv[4] = {hc[u >> 2].x, hc[u >> 2].y, hc[u >> 2].z, hc[u >> 2].w};
#pragma unroll
            for (int t = 0; t < 4; ++t)                                 // m = g ⊙ h̄[s]
              v[u + t] = ex2(fmaf(__uint_as_float(r[u + t]), unL, -mL)) * inv * bv[t];
          }
          // segmented inclusive scan across lanes (fixed tree order)
          for (int d = 1; d < maxlen; d <<= 1) {        // only as many steps as the longest run
#pragma unroll
            for (int u = 0; u < 16; ++u) {
              const float o = __shfl_up_sync(0xffffffffu, v[u], d);
              if (lane - d >= start) v[u] += o;
            }
          }
          if (tail && live) {
            if (!before && !after) {                                   // complete segment
              float *hr = a.h_out + long(tn) * D + cb + c0;
#pragma unroll
              for (int u = 0; u < 16; u += 4) {
                float o4[4];
#pragma unroll
                for (int t = 0; t < 4; ++t) o4[t] = lrelu(a.mean ? v[u + t] / dsc : v[u + t], a.slope);
                *reinterpret_cast<float4 *>(hr + u) = make_float4(o4[0], o4[1], o4[2], o4[3]);
              }
            } else {
              float *pr = a.part + (unit * 2 + (before ? 0 : 1)) * D + cb + c0;
#pragma unroll
              for (int u = 0; u < 16; u += 4)
                *reinterpret_cast<float4 *>(pr + u) = make_float4(v[u], v[u + 1], v[u + 2], v[u + 3]);
            }
          }
        }
      } else
#pragma unroll 1
      for (int c0 = 0; c0 < DH; c0 += 16) {
        uint32_t r[16];
        tc::tmem_ld16(acc + c0, r);
        tc::tmem_ld_wait();
        float o[16];
        if (a.dbg & 8) {
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = __uint_as_float(r[u]) * inv;
        } else {
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = ex2(fmaf(__uint_as_float(r[u]), unL, -mL)) * inv;
        }
        if (!(a.dbg & 2)) warp_store_chunk<D>(wbuf, a.g, wrow0, wrows, cb + c0, o, lane);
      }
      tc::fence_before_sync();
      tc::mbar_arrive(acc2free);
      group_bar(1);        // xg reused by the next tile
    }
    TT_FLUSH_EG(18 + wi);
  }
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  if (warp == 1) tc::tmem_dealloc<TMEM_COLS>(tmem);
}

// ---------------------------------------------------------------------------
// Weight images (built once per parameter update, shared by every row-GEMM launch):
// scale exponent f (max |W|·2^f in [2^14, 2^15)), W·2^f split into fp16 hi / lo in the
// SW128 K-major B-operand layout, [w0 | w1].  One CTA per matrix.
// ---------------------------------------------------------------------------
struct WImageJob {
  const float *W;
  int D, K, transW;
  uint8_t *img;
  int *fexp;
  int bf16;        // OCCU_BF16: one unscaled BF16 image (f = 0) instead of the fp16 pair
};

__global__ void __launch_bounds__(256) wimage_kernel(const WImageJob *__restrict__ jobs) {
  pdl_trigger();
  pdl_wait();
  const WImageJob jb = jobs[blockIdx.x];
  const int D = jb.D, K = jb.K, Kpad = kpad_of(K);
  __shared__ float red[8];
  __shared__ int fe;
  float m = 0.f;
  for (int i = threadIdx.x; i < D * K; i += 256) m = fmaxf(m, fabsf(jb.W[i]));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  // largest row 1-norm of the matrix as used (rows n, columns k): a bound on |W x| for
  // x in [0, 1]^K.  Gate logits W_m e' (e' in (0, 1)) then satisfy |logit| <= bound, and
  // for bound <= 64 the channel softmax needs no max shift (exp cannot overflow or
  // become subnormal; softmax is shift-invariant, so the result is the same function).
  float rs = 0.f;
  for (int n = threadIdx.x; n < D; n += 256) {
    float a = 0.f;
    for (int k = 0; k < K; ++k) a += fabsf(jb.transW ? jb.W[long(k) * D + n] : jb.W[long(n) * K + k]);
    rs = fmaxf(rs, a);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) rs = fmaxf(rs, __shfl_xor_sync(0xffffffffu, rs, o));
  __shared__ float red2[8];
  if ((threadIdx.x & 31) == 0) red2[threadIdx.x >> 5] = rs;
  __syncthreads();
  if (threadIdx.x == 0) {
    float mm = 0.f, rr = 0.f;
    for (int w = 0; w < 8; ++w) {
      mm = fmaxf(mm, red[w]);
      rr = fmaxf(rr, red2[w]);
    }
    fe = jb.bf16 ? 0 : scale_exp(mm);
    jb.fexp[0] = fe;
    jb.fexp[1] = rr <= 64.f ? 1 : 0;
  }
  __syncthreads();
  const float ws = ldexpf(1.f, fe);
  const uint32_t ib = uint32_t(Kpad) * D * 2;
  for (int i = threadIdx.x; i < D * (Kpad / 2); i += 256) {
    const int n = i / (Kpad / 2), k = 2 * (i % (Kpad / 2));
    const long i0 = jb.transW ? long(k) * D + n : long(n) * K + k;
    const long i1 = jb.transW ? long(k + 1) * D + n : long(n) * K + k + 1;
    const float v0 = k < K ? jb.W[i0] * ws : 0.f;
    const float v1 = k + 1 < K ? jb.W[i1] * ws : 0.f;
    const uint32_t off = tc::sw128_offset_f16(n, k, D);
    if (jb.bf16) {
      const __nv_bfloat162 b = __floats2bfloat162_rn(v0, v1);
      *reinterpret_cast<__nv_bfloat162 *>(jb.img + off) = b;
    } else {
      uint32_t hi, lo;
      split2(v0, v1, hi, lo);
      *reinterpret_cast<uint32_t *>(jb.img + off) = hi;
      *reinterpret_cast<uint32_t *>(jb.img + ib + off) = lo;
    }
  }
}

// Layer-1 edge transform (F_e small, e.g. 4): e' = σ(α · W_e e) on CUDA cores (a3).
// A warp takes 32 consecutive in-CSR edges per iteration: lane j loads edge j's
// indices, α = p[src] + q[dst] and its Ke input features (one independent gather
// chain per lane, all 32 in flight), then the warp walks the 32 edges, broadcasting
// α and e by shuffle; each lane computes D/32 channels of the edge's row
// (coalesced row stores).  With eid != null the input row of in-CSR edge k is
// e_in[eid[k]] (a1's permutation fused in); e0_out, if set, receives the permuted
// rows (kept for the backward).  Ke <= KM <= 16.
template <int D, int KM>
__global__ void __launch_bounds__(256) edge_small_kernel(
    const float *__restrict__ e_in, int Ke, const float *__restrict__ W_e,
    const float *__restrict__ p, const float *__restrict__ q, const int32_t *__restrict__ in_src,
    const int32_t *__restrict__ in_dst, const int32_t *__restrict__ eid, int E,
    float *__restrict__ e_out, float *__restrict__ e0_out) {
  constexpr int V = D / 32;                 // channels per lane
  extern __shared__ float wsm[];            // [Ke][D] = W_eᵀ
  pdl_trigger();
  pdl_wait();
  for (int i = threadIdx.x; i < D * Ke; i += blockDim.x) wsm[(i % Ke) * D + i / Ke] = W_e[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int c = lane * V;
  float w[KM][V];                           // this lane's W_e columns, in registers
#pragma unroll
  for (int j = 0; j < KM; ++j)
#pragma unroll
    for (int v = 0; v < V; ++v) w[j][v] = j < Ke ? wsm[j * D + c + v] : 0.f;
  const long nwarps = long(gridDim.x) * (blockDim.x / 32);
  for (long k0 = (blockIdx.x * long(blockDim.x / 32) + threadIdx.x / 32) * 32; k0 < E;
       k0 += nwarps * 32) {
    const long k = k0 + lane;
    const int cnt = int(min(32L, E - k0));
    float al = 0.f, ev[KM];
#pragma unroll
    for (int j = 0; j < KM; ++j) ev[j] = 0.f;
    if (k < E) {
      al = __ldg(p + __ldg(in_src + k)) + __ldg(q + __ldg(in_dst + k));
      const long row = eid ? long(__ldg(eid + k)) : k;
      if (KM == 4 && Ke == 4) {
        const float4 x = __ldg(reinterpret_cast<const float4 *>(e_in + row * 4));
        ev[0] = x.x; ev[1 % KM] = x.y; ev[2 % KM] = x.z; ev[3 % KM] = x.w;
      } else {
#pragma unroll
        for (int j = 0; j < KM; ++j) ev[j] = j < Ke ? __ldg(e_in + row * Ke + j) : 0.f;
      }
      if (e0_out) {
#pragma unroll
        for (int j = 0; j < KM; ++j)
          if (j < Ke) e0_out[k * Ke + j] = ev[j];
      }
    }
    for (int u = 0; u < cnt; ++u) {
      const float a = __shfl_sync(0xffffffffu, al, u);
      float z[V];
#pragma unroll
      for (int v = 0; v < V; ++v) z[v] = 0.f;
#pragma unroll
      for (int j = 0; j < KM; ++j) {
        const float x = __shfl_sync(0xffffffffu, ev[j], u);
#pragma unroll
        for (int v = 0; v < V; ++v) z[v] = fmaf(w[j][v], x, z[v]);
      }
      float o[V];
#pragma unroll
      for (int v = 0; v < V; ++v) o[v] = fast_rcp(1.f + fast_exp(-(a * z[v])));
      float *dst = e_out + (k0 + u) * D + c;
      if constexpr (V == 4) {
        *reinterpret_cast<float4 *>(dst) = make_float4(o[0], o[1], o[2], o[3]);
      } else if constexpr (V == 8) {
        *reinterpret_cast<float4 *>(dst) = make_float4(o[0], o[1], o[2], o[3]);
        *reinterpret_cast<float4 *>(dst + 4) = make_float4(o[4 % V], o[5 % V], o[6 % V], o[7 % V]);
      } else {
#pragma unroll
        for (int v = 0; v < V; v += 2) *reinterpret_cast<float2 *>(dst + v) = make_float2(o[v], o[v + 1]);
      }
    }
  }
}

// ---------------------------------------------------------------------------
// Weight gradients on tensor cores: partial[split][a][b] = Σ_{r in split} X[r][a] Y[r][b]
// (dW_m = DVᵀE', dW_e = DZᵀE_in, dW_u = dPᵀH_in; SURVEY §8(c) step BW).  3xTF32 with
// the MMA's own tf32 truncation as the "hi" part: hi = X (raw fp32 in smem), lo =
// X - trunc13(X) computed in smem; X and Y tiles arrive by 2D TMA (32 rows x 32 columns
// SW128 boxes) and are consumed as MN-major operands (M = a, N = b, K = row).  Each CTA
// owns a contiguous row range; partials are reduced in fixed split order afterwards.
// ---------------------------------------------------------------------------
// YBF (OCCU_BF16 training, R28): Y rows are BF16.  TMA lands them (32 rows x 64 bf16 SW128
// boxes) in the Y-lo region; the lo warps widen them (exactly) into the Y raw region, and
// since a BF16 value is its own tf32 hi part (Y lo = 0) the X_hi·Y_lo product is skipped.
constexpr int WG_ROWS = 32;               // rows (K) per pipeline stage
constexpr int WG_NS = 3;                  // pipeline stages (16-row x 6 and 2 CTAs/SM measured slower)
constexpr int WG_BOX = WG_ROWS * 128;     // one TMA box: WG_ROWS rows x 32 fp32 (or 64 bf16)
constexpr int WG_REG = 4 * WG_BOX;        // one operand region (4 boxes = 128 columns)
constexpr int WG_STAGE = 4 * WG_REG;      // X raw, X lo, Y raw, Y lo
constexpr int WG_Q4 = WG_ROWS * 8;        // float4 per box
constexpr int WG_IT = 2 * 4 * WG_Q4 / 256;  // float4 per lo-warp thread per stage
constexpr int WG_NTH = 320;               // warp0 TMA, warp1 MMA, warps 2-9 lo / epilogue

// Logical 16-byte chunk stored at physical slot pc of 128-byte row r under the TMA
// SWIZZLE_128B_ATOM_32B pattern (32-byte chunks permuted: chunk32 ^ (r & 3)).
__device__ __forceinline__ int wg_logical_chunk(int pc, int r) {
  return ((((pc >> 1) ^ (r & 3))) << 1) | (pc & 1);
}

template <bool YBF>
__global__ void __launch_bounds__(WG_NTH, 1)
wgrad_tc_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap ymap,
                int A, int Bn, long R, int splits, float *__restrict__ partial) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t sa = tc::smem_u32(smem_raw);
  uint8_t *base = smem_raw + ((1024 - (sa & 1023)) & 1023);
  // stage s: X raw (4 boxes of WG_ROWS rows x 128 B), X lo, Y raw, Y lo (Y-lo region = BF16
  // landing zone when YBF)
  auto stage = [&](int s2) { return base + s2 * WG_STAGE; };
  uint64_t *bars = reinterpret_cast<uint64_t *>(base + WG_NS * WG_STAGE);
  uint64_t *full = bars, *lo_ready = bars + WG_NS, *empty = bars + 2 * WG_NS, *done = bars + 3 * WG_NS;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * WG_NS + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nbx = (A + 31) / 32, nby = (Bn + 31) / 32, nbyb = (Bn + 63) / 64;
  const int Npad = (Bn + 15) / 16 * 16;
  // zero every box region once: boxes that TMA never writes (A or B < 128) stay zero
  for (int i = threadIdx.x; i < WG_NS * WG_STAGE / 16; i += WG_NTH)
    reinterpret_cast<float4 *>(base)[i] = make_float4(0.f, 0.f, 0.f, 0.f);
  if (threadIdx.x == 0) {
    for (int j = 0; j < WG_NS; ++j) {
      tc::mbar_init(full + j, 1);
      tc::mbar_init(lo_ready + j, 256);
      tc::mbar_init(empty + j, 1);
    }
    tc::mbar_init(done, 1);
    tc::fence_mbar_init();
  }
  if (warp == 1) tc::tmem_alloc<128>(tmem_slot);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  const uint32_t tmem = *tmem_slot;
  const long per = (R + splits - 1) / splits;
  const long rb = blockIdx.x * per, re = min(R, rb + per);
  const int nst = rb < re ? int((re - rb + WG_ROWS - 1) / WG_ROWS) : 0;

  if (warp == 0) {
    if (lane == 0) {
      tc::prefetch_tmap(&xmap);
      tc::prefetch_tmap(&ymap);
      for (int i = 0; i < nst; ++i) {
        const int j = i % WG_NS;
        if (i >= WG_NS) tc::mbar_wait(empty + j, ((i / WG_NS) - 1) & 1);
        const int r0 = int(rb + long(i) * WG_ROWS);
        uint8_t *st = stage(j);
        tc::mbar_arrive_expect_tx(full + j, uint32_t(nbx + (YBF ? nbyb : nby)) * uint32_t(WG_BOX));
        for (int b = 0; b < nbx; ++b) tc::tma_load_2d(st + b * WG_BOX, &xmap, 32 * b, r0, full + j);
        if (YBF)
          for (int b = 0; b < nbyb; ++b) tc::tma_load_2d(st + 3 * WG_REG + b * WG_BOX, &ymap, 64 * b, r0, full + j);
        else
          for (int b = 0; b < nby; ++b) tc::tma_load_2d(st + 2 * WG_REG + b * WG_BOX, &ymap, 32 * b, r0, full + j);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    const uint32_t idsc = tc::idesc(128, uint32_t(Npad), tc::FMT_TF32) | (1u << 15) | (1u << 16);
    for (int i = 0; i < nst; ++i) {
      const int j = i % WG_NS;
      tc::mbar_wait(lo_ready + j, (i / WG_NS) & 1);
      tc::fence_after_sync();
      if (lane == 0) {
        const uint32_t st = tc::smem_u32(stage(j));
        for (int kg = 0; kg < WG_ROWS / 8; ++kg) {
          const uint64_t ah = tc::sdesc_sw128b32_mn(st + kg * 1024, WG_BOX);
          const uint64_t al = tc::sdesc_sw128b32_mn(st + WG_REG + kg * 1024, WG_BOX);
          const uint64_t bh = tc::sdesc_sw128b32_mn(st + 2 * WG_REG + kg * 1024, WG_BOX);
          const uint64_t bl = tc::sdesc_sw128b32_mn(st + 3 * WG_REG + kg * 1024, WG_BOX);
          tc::mma_tf32_ss(tmem, ah, bh, idsc, (i > 0 || kg > 0) ? 1u : 0u);
          if (!YBF) tc::mma_tf32_ss(tmem, ah, bl, idsc, 1u);
          tc::mma_tf32_ss(tmem, al, bh, idsc, 1u);
        }
        tc::mma_commit(empty + j);
        if (i == nst - 1) tc::mma_commit(done);
      }
      __syncwarp();
    }
  } else {
    const int t = threadIdx.x - 64;              // 0..255
    for (int i = 0; i < nst; ++i) {
      const int j = i % WG_NS;
      tc::mbar_wait(full + j, (i / WG_NS) & 1);
      uint8_t *st = stage(j);
      const long r0 = rb + long(i) * WG_ROWS;
      // X raw -> X lo (boxes 0..nbx), Y raw -> Y lo; rows beyond this CTA's range -> 0.
      // 2 operands x 4 boxes x WG_ROWS·8 float4 = WG_IT per thread, all loads issued first.
      float4 v[WG_IT];
#pragma unroll
      for (int it = 0; it < WG_IT; ++it) {
        const int f = t + it * 256, op = f / (4 * WG_Q4), b = (f / WG_Q4) & 3, q4 = f % WG_Q4;
        v[it] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (b < (op == 0 ? nbx : nby)) {
          if (YBF && op == 1) {
            // fp32 box b (SWIZZLE_128B_ATOM_32B), row rr, physical 16-byte slot q4 & 7 holds
            // logical chunk c (columns 32b+4c..+3) <- bf16 box b/2 (plain SW128: chunk ^ (row & 7)),
            // logical chunk 4(b&1) + c/2, half c&1
            const int rr = q4 >> 3, c = wg_logical_chunk(q4 & 7, rr), cb = 4 * (b & 1) + (c >> 1);
            const uint2 w = *reinterpret_cast<const uint2 *>(st + 3 * WG_REG + (b >> 1) * WG_BOX + rr * 128 +
                                                             ((cb ^ (rr & 7)) << 4) + (c & 1) * 8);
            v[it] = make_float4(__uint_as_float(w.x << 16), __uint_as_float(w.x & 0xFFFF0000u),
                                __uint_as_float(w.y << 16), __uint_as_float(w.y & 0xFFFF0000u));
          } else {
            v[it] = reinterpret_cast<const float4 *>(st + op * 2 * WG_REG + b * WG_BOX)[q4];
          }
        }
      }
#pragma unroll
      for (int it = 0; it < WG_IT; ++it) {
        const int f = t + it * 256, op = f / (4 * WG_Q4), b = (f / WG_Q4) & 3, q4 = f % WG_Q4;
        if (b >= (op == 0 ? nbx : nby)) continue;
        float4 x = v[it];
        if (YBF && op == 1) {                             // widened BF16 row: raw, no lo
          if (r0 + (q4 >> 3) >= re) x = make_float4(0.f, 0.f, 0.f, 0.f);
          reinterpret_cast<float4 *>(st + 2 * WG_REG + b * WG_BOX)[q4] = x;
          continue;
        }
        if (r0 + (q4 >> 3) >= re) {                       // 8 float4 per 128-byte row
          x = make_float4(0.f, 0.f, 0.f, 0.f);
          reinterpret_cast<float4 *>(st + op * 2 * WG_REG + b * WG_BOX)[q4] = x;
        }
        float4 l;
        l.x = x.x - __uint_as_float(__float_as_uint(x.x) & 0xFFFFE000u);
        l.y = x.y - __uint_as_float(__float_as_uint(x.y) & 0xFFFFE000u);
        l.z = x.z - __uint_as_float(__float_as_uint(x.z) & 0xFFFFE000u);
        l.w = x.w - __uint_as_float(__float_as_uint(x.w) & 0xFFFFE000u);
        reinterpret_cast<float4 *>(st + op * 2 * WG_REG + WG_REG + b * WG_BOX)[q4] = l;
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      tc::mbar_arrive(lo_ready + j);
    }
    // epilogue: thread = output row a (TMEM lane), columns b
    if (nst > 0) {
      tc::mbar_wait(done, 0);
      tc::fence_after_sync();
    }
    const int q = warp & 3, row = q * 32 + lane, hh = (warp - 2) >> 2;
    const uint32_t lane_base = tmem + (uint32_t(q * 32) << 16);
    float *out = partial + long(blockIdx.x) * A * Bn + long(row) * Bn;
    const int chalf = (Npad / 16 + 1) / 2 * 16;             // two warps per TMEM lane quarter
    for (int c0 = hh * chalf; c0 < min(Npad, (hh + 1) * chalf); c0 += 16) {
      uint32_t r[16];
      if (nst > 0) {
        tc::tmem_ld16(lane_base + c0, r);
        tc::tmem_ld_wait();
      } else {
#pragma unroll
        for (int u = 0; u < 16; ++u) r[u] = 0u;
      }
      if (row < A)
#pragma unroll
        for (int u = 0; u < 16; ++u)
          if (c0 + u < Bn) out[c0 + u] = __uint_as_float(r[u]);
    }
  }
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  if (warp == 1) tc::tmem_dealloc<128>(tmem);
}

typedef CUresult (*PFN_encodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                    const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                    const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                    CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// Tensor map of a row-major fp32 matrix [R][K]: boxes of 128 rows x 32 columns,
// 128-byte swizzle, out-of-bounds elements read as zero.
bool encode_rows_map(CUtensorMap *m, const float *A, int R, int K) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !p)
      return false;
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  const cuuint64_t dims[2] = {cuuint64_t(K), cuuint64_t(R)};
  const cuuint64_t strides[1] = {cuuint64_t(K) * 4};
  const cuuint32_t box[2] = {32, 128};
  const cuuint32_t estr[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(A), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Nodes whose in-edge segment spans several 32-edge units: combine the fixed-slot
// partials in unit order; nodes without in-edges: h = LReLU(0) = 0 (R8).
__global__ void agg_fixup_kernel(const int32_t *__restrict__ in_ptr, int N, int D,
                                 const float *__restrict__ part, int mean, float slope,
                                 float *__restrict__ h_out) {
  const int warps = (gridDim.x * blockDim.x) / 32;
  const int lane = threadIdx.x & 31;
  for (int t0 = (blockIdx.x * blockDim.x + threadIdx.x) / 32 * 32; t0 < N; t0 += warps * 32) {
    const int t = t0 + lane;
    int beg = 0, end = 0;
    if (t < N) {
      beg = in_ptr[t];
      end = in_ptr[t + 1];
    }
    const bool special = t < N && (beg == end || (beg >> 5) != ((end - 1) >> 5));
    unsigned m = __ballot_sync(0xffffffffu, special);
    while (m) {                                      // warp-cooperative over channels
      const int l = __ffs(m) - 1;
      m &= m - 1;
      const int tt = t0 + l;
      const int b2 = __shfl_sync(0xffffffffu, beg, l), e2 = __shfl_sync(0xffffffffu, end, l);
      for (int c = lane; c < D; c += 32) {
        float v = 0.f;
        if (b2 != e2) {
          const int ub = b2 >> 5, ue = (e2 - 1) >> 5;
          v = part[(long(ub) * 2 + 1) * D + c];
          for (int u = ub + 1; u <= ue; ++u) v += part[(long(u) * 2 + 0) * D + c];
          if (mean) v = v / float(e2 - b2);
        }
        h_out[long(tt) * D + c] = lrelu(v, slope);
      }
    }
  }
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

static bool encode_rows_map32(CUtensorMap *m, const float *A, long R, int K) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !p)
      return false;
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  const cuuint64_t dims[2] = {cuuint64_t(K), cuuint64_t(R)};
  const cuuint64_t strides[1] = {cuuint64_t(K) * 4};
  const cuuint32_t box[2] = {32, WG_ROWS};
  const cuuint32_t estr[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(A), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// BF16 rows [R][K]: boxes of 32 rows x 64 bf16 (128 B), 128-byte swizzle, OOB zero.
static bool encode_rows_map32_bf16(CUtensorMap *m, const void *A, long R, int K) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !p)
      return false;
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  const cuuint64_t dims[2] = {cuuint64_t(K), cuuint64_t(R)};
  const cuuint64_t strides[1] = {cuuint64_t(K) * 2};
  const cuuint32_t box[2] = {64, WG_ROWS};
  const cuuint32_t estr[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(A), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Bn < 16 or not a multiple of 16 (e.g. dW_e of layer 1, F_e = 4): the TMA box reads the
// missing columns as zeros (out of bounds) and the MMA runs N = Bn rounded up to 16.
bool wgrad_tc_supported(int A, int Bn) {
  return A >= 32 && A <= 128 && A % 32 == 0 && Bn >= 4 && Bn <= 128 && Bn % 4 == 0;
}

// partial must hold splits * A * Bn floats; returns the number of launches (1) or -err.
int launch_wgrad_tc(const occu_ctx *ctx, const float *X, int A, const void *Y, int Bn, long R,
                    int splits, float *partial, cudaStream_t st, bool ybf) {
  CUtensorMap xm, ym;
  if (!encode_rows_map32(&xm, X, R, A) ||
      !(ybf ? encode_rows_map32_bf16(&ym, Y, R, Bn) : encode_rows_map32(&ym, static_cast<const float *>(Y), R, Bn)))
    return -int(cudaErrorInvalidValue);
  const size_t smem = 1024 + size_t(WG_NS) * WG_STAGE + 256;
  OCCU_PROF_BEGIN(ctx, "wgrad_tc", st);
  if (ybf) {
    set_smem(wgrad_tc_kernel<true>, smem);
    wgrad_tc_kernel<true><<<splits, WG_NTH, smem, st>>>(xm, ym, A, Bn, R, splits, partial);
  } else {
    set_smem(wgrad_tc_kernel<false>, smem);
    wgrad_tc_kernel<false><<<splits, WG_NTH, smem, st>>>(xm, ym, A, Bn, R, splits, partial);
  }
  OCCU_PROF_END(ctx);
  TC_CHECK();
  return 1;
}

// one image slot: [w0 | w1], Kpad <= 128 and D <= 128; at d = 256 Kpad, D <= 256
static size_t wimg_slot_bytes(const occu_config &c) {
  return c.d > 128 ? size_t(2) * 256 * 256 * 2 : size_t(2) * 128 * 128 * 2;
}

const uint8_t *tc_wimg(const occu_ctx *ctx, int kind, int layer) {
  return ctx->wimg.as<uint8_t>() + size_t(layer * 6 + kind) * wimg_slot_bytes(ctx->cfg);
}
const int *tc_wfexp(const occu_ctx *ctx, int kind, int layer) {
  return ctx->wfexp.as<int>() + (layer * 6 + kind) * 2;     // [f, softmax no-shift flag]
}

// (Re)build the images when the parameters changed (set_params / Adam bump the version).
int tc_prepare_weights(occu_ctx *ctx, cudaStream_t st) {
  if (ctx->wimg_version == ctx->params_version) return 0;
  const occu_config &c = ctx->cfg;
  const ParamLayout &L = ctx->layout;
  // slots: 6 kinds per ANEE layer, plus "layer" L for the decoder's FFN (kinds 0, 1) and
  // "layer" L + 1 + j for Graphormer layer j (kinds 0-5: W_q, W_k, W_v, W_o, FFN W1, W2)
  // + "layer" L + 1 + G + j: Graphormer layer j's transposed matrices (backward, gph_tslot)
  const size_t nslot = size_t(c.L + 1 + 2 * c.graphormer) * 6;
  const int kmax = c.d > 128 ? 256 : 128;     // largest K an image slot holds
  if (ctx->wimg.ensure(nslot * wimg_slot_bytes(c)) != cudaSuccess ||
      ctx->wfexp.ensure(nslot * 2 * sizeof(int)) != cudaSuccess ||
      ctx->wjobs.ensure(nslot * sizeof(WImageJob)) != cudaSuccess)
    return -int(cudaErrorMemoryAllocation);
  std::vector<WImageJob> jobs;
  const float *P = ctx->params.as<float>();
  for (int i = 0; i < c.L; ++i) {
    auto add = [&](int kind, const float *W, int D, int K, int transW) {
      WImageJob j;
      j.W = W; j.D = D; j.K = K; j.transW = transW;
      // OCCU_BF16: the forward images (kinds 0-2) are BF16; the backward images (3-5) multiply
      // FP32 gradients and stay fp16x2 FP32 images (R28)
      j.bf16 = c.prec == OCCU_BF16 && kind <= 2;
      j.img = const_cast<uint8_t *>(tc_wimg(ctx, kind, i));
      j.fexp = const_cast<int *>(tc_wfexp(ctx, kind, i));
      jobs.push_back(j);
    };
    const bool fwd_only = c.d > 128;     // d = 256 runs inference only (no backward images)
    if (L.d_in[i] <= kmax) add(0, P + L.W_u[i], c.d, L.d_in[i], 0);
    if (L.de_in[i] > 16 && L.de_in[i] <= kmax) {
      add(1, P + L.W_e[i], c.d, L.de_in[i], 0);
      if (!fwd_only) add(4, P + L.W_e[i], c.d, c.d, 1);
    }
    add(2, P + L.W_m[i], c.d, c.d, 0);
    if (!fwd_only) add(3, P + L.W_m[i], c.d, c.d, 1);
    if (i > 0 && !fwd_only) add(5, P + L.W_u[i], c.d, c.d, 1);
  }
  if (L.dec) {      // NEXT-2 decoder: the pre-pooling FFN's two d x d matrices
    auto addd = [&](int kind, const float *W, int transW = 0) {
      WImageJob j;
      j.W = W; j.D = c.d; j.K = c.d; j.transW = transW; j.bf16 = 0;
      j.img = const_cast<uint8_t *>(tc_wimg(ctx, kind, c.L));
      j.fexp = const_cast<int *>(tc_wfexp(ctx, kind, c.L));
      jobs.push_back(j);
    };
    addd(0, P + L.D.P.W1);
    addd(1, P + L.D.P.W2);
    addd(2, P + L.D.P.W1, 1);           // transposed (training: dX = dY·W)
    addd(3, P + L.D.P.W2, 1);
  }
  for (int j = 0; j < c.graphormer; ++j) {      // NEXT-3 Graphormer: six d x d matrices
    const GphOff &g = L.G[j];
    const size_t ws[6] = {g.Wq, g.Wk, g.Wv, g.Wo, g.F.W1, g.F.W2};
    for (int kind = 0; kind < 6; ++kind) {
      WImageJob jb;
      jb.W = P + ws[kind]; jb.D = c.d; jb.K = c.d; jb.transW = 0; jb.bf16 = 0;
      jb.img = const_cast<uint8_t *>(tc_wimg(ctx, kind, c.L + 1 + j));
      jb.fexp = const_cast<int *>(tc_wfexp(ctx, kind, c.L + 1 + j));
      jobs.push_back(jb);
      jb.transW = 1;                   // dX = dY·W of the backward
      jb.img = const_cast<uint8_t *>(tc_wimg(ctx, kind, gph_tslot(c, j)));
      jb.fexp = const_cast<int *>(tc_wfexp(ctx, kind, gph_tslot(c, j)));
      jobs.push_back(jb);
    }
  }
  // job table: pointers are fixed for the ctx, re-uploaded only with the images
  if (cudaMemcpyAsync(ctx->wjobs.ptr, jobs.data(), jobs.size() * sizeof(WImageJob),
                      cudaMemcpyHostToDevice, st) != cudaSuccess)
    return -int(cudaErrorInvalidValue);
  OCCU_PROF_BEGIN(ctx, "wimage", st);
  launch_pdl(ctx->pdl & 32, wimage_kernel, int(jobs.size()), 256, 0, st, ctx->wjobs.as<WImageJob>());
  OCCU_PROF_END(ctx);
  TC_CHECK();
  ctx->wimg_version = ctx->params_version;
  return 1;
}

int gph_tslot(const occu_config &c, int j) { return c.L + 1 + c.graphormer + j; }

bool tc_supported(const occu_config &c) {
  return ((c.d == 64 || c.d == 128) && c.F_n <= 128) || (c.d == 256 && c.F_n <= 256);
}

size_t tc_partial_floats(int E, int D) { return size_t(E / 32 + 2) * 2 * D; }

template <int D, int EPI>
static int launch_rowgemm(const occu_ctx *ctx, const RowGemmArgs &ra, const char *name,
                          cudaStream_t st) {
  if (ra.R <= 0) return 0;
  const size_t smem = smem_bytes(D, ra.K);
  set_smem(rowgemm_kernel<D, EPI>, smem);
  const int tiles = (ra.R + TM - 1) / TM;
  const int grid = std::min(tiles, ctx->num_sms);
  CUtensorMap tmap;
  if (!encode_rows_map(&tmap, ra.A, ra.R, ra.K)) return -int(cudaErrorInvalidValue);
  static const int dot2 = [] {
    const char *e = getenv("OCCU_DA_F64");
    return e && atoi(e) ? 0 : 1;
  }();
  RowGemmArgs rc = ra;
  rc.dot2 = dot2;
  OCCU_PROF_BEGIN(ctx, name, st);
  launch_pdl(ctx->pdl & 1, rowgemm_kernel<D, EPI>, grid, NTH, smem, st, tmap, rc);
  OCCU_PROF_END(ctx);
  TC_CHECK();
  return 1;
}

// BF16 rows [R][K]: boxes of 128 rows x 64 bf16 (128 B), 128-byte swizzle, OOB zero
static bool encode_rows_map_bf16_128(CUtensorMap *m, const void *A, long R, int K) {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !p)
      return false;
    fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  const cuuint64_t dims[2] = {cuuint64_t(K), cuuint64_t(R)};
  const cuuint64_t strides[1] = {cuuint64_t(K) * 2};
  const cuuint32_t box[2] = {64, 128};
  const cuuint32_t estr[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(A), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// d = 256: CTA-pair row-GEMM (rowgemm_pair_kernel), grid = 2 x clusters.  FP32 mode (BF =
// false): FP32 rows, per-row scale exponents for node inputs first (row_exp_kernel).
template <int EPI, bool BF, bool AF32>
static int launch_rowgemm_pair(const occu_ctx *ctx, RowGemmArgs ra, const char *name,
                               cudaStream_t st) {
  static_assert(BF || AF32, "OCCU_FP32 rows are FP32");
  if (ra.R <= 0) return 0;
  if (ra.K > 256 || (!AF32 && ra.K % 64)) return -int(cudaErrorInvalidValue);
  const size_t smem = pair_smem_bytes(ra.K, BF ? 1 : 2);
  set_smem(rowgemm_pair_kernel<EPI, BF, AF32>, smem);
  const int tiles = (ra.R + 2 * TM - 1) / (2 * TM);
  const int clusters = std::max(1, std::min(tiles, ctx->num_sms / 2));
  CUtensorMap tmap;
  if (!(AF32 ? encode_rows_map(&tmap, ra.A, ra.R, ra.K) : encode_rows_map_bf16_128(&tmap, ra.A, ra.R, ra.K)))
    return -int(cudaErrorInvalidValue);
  int n = 0;
  OCCU_PROF_BEGIN(ctx, name, st);
  ra.rexp = nullptr;
  if (!BF && EPI == EPI_NODE && (ra.K + 31) / 32 > P_NS) {   // K > 128: the rows' scale exponents first
    if (const_cast<occu_ctx *>(ctx)->ws.rowexp.ensure(size_t(ra.R) * 4) != cudaSuccess)
      return -int(cudaErrorMemoryAllocation);
    int *rexp = ctx->ws.rowexp.as<int>();
    ra.rexp = rexp;
    const int g = int(std::min<long>((long(ra.R) + 7) / 8, 16L * ctx->num_sms));
    launch_pdl(ctx->pdl & 1, row_exp_kernel, g, 256, 0, st, ra.A, ra.R, ra.K, rexp);
    ++n;
  }
  launch_pdl(ctx->pdl & 1, rowgemm_pair_kernel<EPI, BF, AF32>, 2 * clusters, P_NTH, smem, st, tmap, ra);
  OCCU_PROF_END(ctx);
  TC_CHECK();
  return n + 1;
}

// One ANEE layer at d = 256 (a2-a6), FP32: node transform, edge transform (CUDA cores for
// F_e <= 16, else the pair GEMM), channel-softmax gate, then the CUDA-core aggregation.
static int tc_forward_layer_pair(const occu_ctx *ctx, const DevCsr &csr, int layer,
                                 const FwdLayerArgs &a, cudaStream_t st) {
  constexpr int D = 256;
  const float slope = ctx->cfg.slope;
  int n = 0, r;
  RowGemmArgs ra{};
  ra.slope = slope;
  ra.A = a.h_in; ra.K = a.K; ra.R = csr.N; ra.W = a.W_u; ra.out = a.hbar;
  ra.wimg = tc_wimg(ctx, 0, layer); ra.wfexp = tc_wfexp(ctx, 0, layer);
  ra.a_s = a.a_s; ra.a_d = a.a_d; ra.p = a.p; ra.q = a.q;
  ra.rev = ctx->l2_order;
  if ((r = launch_rowgemm_pair<EPI_NODE, false, true>(ctx, ra, "node_tc", st)) < 0) return r;
  n += r;
  if (csr.E > 0) {
    if (a.Ke <= 16) {
      const int grid = int(std::min<long>((long(csr.E) + 255) / 256, 8L * ctx->num_sms));
      OCCU_PROF_BEGIN(ctx, "edge_small", st);
      if (a.Ke <= 4)
        launch_pdl(ctx->pdl & 4, edge_small_kernel<D, 4>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke, a.W_e,
                   a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, a.e_out, a.e0_out);
      else
        launch_pdl(ctx->pdl & 4, edge_small_kernel<D, 16>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke, a.W_e,
                   a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, a.e_out, a.e0_out);
      OCCU_PROF_END(ctx);
      TC_CHECK();
      ++n;
    } else {
      RowGemmArgs re{};
      re.slope = slope;
      re.A = a.e_in; re.K = a.Ke; re.R = csr.E; re.W = a.W_e; re.out = a.e_out;
      re.wimg = tc_wimg(ctx, 1, layer); re.wfexp = tc_wfexp(ctx, 1, layer);
      re.pin = a.p; re.qin = a.q; re.src = csr.in_src; re.dst = csr.in_dst;
      if ((r = launch_rowgemm_pair<EPI_EDGE, false, true>(ctx, re, "edge_tc", st)) < 0) return r;
      n += r;
    }
    RowGemmArgs rg{};
    rg.slope = slope;
    rg.A = a.e_out; rg.K = D; rg.R = csr.E; rg.W = a.W_m; rg.out = a.g;
    rg.wimg = tc_wimg(ctx, 2, layer); rg.wfexp = tc_wfexp(ctx, 2, layer);
    rg.rev = ctx->l2_order;
    if ((r = launch_rowgemm_pair<EPI_GATE, false, true>(ctx, rg, "gate_tc", st)) < 0) return r;
    n += r;
  }
  if ((r = launch_gather_segsum(ctx, csr, a.g, a.hbar, a.h_out, a.rpart, st, a.h_bits)) < 0) return r;
  return n + r;
}

template <int D>
static int launch_edgegate(const occu_ctx *ctx, const DevCsr &csr, int layer, const FwdLayerArgs &a,
                           cudaStream_t st, float *partial = nullptr) {
  if (csr.E <= 0) return 0;
  const bool first = a.Ke <= 16;
  const bool agg = partial != nullptr;
  EdgeGateArgs ea{};
  ea.hbar = a.hbar; ea.in_ptr = csr.in_ptr; ea.h_out = a.h_out; ea.part = partial;
  ea.mean = ctx->cfg.aggr == OCCU_AGGR_MEAN; ea.slope = ctx->cfg.slope;
  ea.e_in = a.e_in; ea.Ke = a.Ke; ea.R = csr.E; ea.eid = a.e_eid; ea.W_e = a.W_e;
  ea.wimg_m = tc_wimg(ctx, 2, layer); ea.wf_m = tc_wfexp(ctx, 2, layer);
  if (!first) {
    ea.wimg_e = tc_wimg(ctx, 1, layer);
    ea.wf_e = tc_wfexp(ctx, 1, layer);
  }
  ea.p = a.p; ea.q = a.q; ea.src = csr.in_src; ea.dst = csr.in_dst;
  ea.e_out = a.e_out; ea.e0_out = a.e0_out; ea.g = a.g;
  ea.rev = ctx->l2_order;
  static const int dbg = [] {
    const char *e = getenv("OCCU_EG_DBG");
    return e ? atoi(e) : 0;
  }();
  ea.dbg = dbg;
  const size_t smem = eg_smem_bytes(D, a.Ke, first);
  const int tiles = (csr.E + TM - 1) / TM;
  const int grid = std::min(tiles, ctx->num_sms);
  CUtensorMap tmap;
  memset(&tmap, 0, sizeof(tmap));
  if (!first && !encode_rows_map(&tmap, a.e_in, csr.E, a.Ke)) return -int(cudaErrorInvalidValue);
  OCCU_PROF_BEGIN(ctx, agg ? "edge_gate_agg_tc" : "edge_gate_tc", st);
#define OCCU_EG_LAUNCH(KMV, AGGV)                                                   \
  do {                                                                            \
    set_smem(edgegate_kernel<D, KMV, AGGV>, smem);                                \
    edgegate_kernel<D, KMV, AGGV><<<grid, EG_NTH, smem, st>>>(tmap, ea);           \
  } while (0)
  if (!first) {
    if (agg) OCCU_EG_LAUNCH(0, true); else OCCU_EG_LAUNCH(0, false);
  } else if (a.Ke <= 4) {
    if (agg) OCCU_EG_LAUNCH(4, true); else OCCU_EG_LAUNCH(4, false);
  } else {
    if (agg) OCCU_EG_LAUNCH(16, true); else OCCU_EG_LAUNCH(16, false);
  }
#undef OCCU_EG_LAUNCH
  OCCU_PROF_END(ctx);
  TC_CHECK();
  return 1;
}

template <int D>
static int tc_forward_layer_impl(const occu_ctx *ctx, const DevCsr &csr, int layer,
                                 const FwdLayerArgs &a, float *partial, cudaStream_t st) {
  const float slope = ctx->cfg.slope;
  int n = 0, r;
  RowGemmArgs ra{};
  ra.slope = slope;
  // a2: node transform
  ra.A = a.h_in; ra.K = a.K; ra.R = csr.N; ra.W = a.W_u; ra.out = a.hbar;
  ra.wimg = tc_wimg(ctx, 0, layer); ra.wfexp = tc_wfexp(ctx, 0, layer);
  ra.a_s = a.a_s; ra.a_d = a.a_d; ra.p = a.p; ra.q = a.q;
  // L2 reuse: node and gate walk their rows last-to-first, so each kernel starts on the
  // rows its producer (gather resp. edge transform, both first-to-last) wrote last
  ra.rev = ctx->l2_order;
  if ((r = launch_rowgemm<D, EPI_NODE>(ctx, ra, "node_tc", st)) < 0) return r;
  n += r;
  const bool eg_shape = ctx->path == 0 && ctx->cfg.msg == OCCU_MSG_CHANNEL_SOFTMAX &&
                        (a.Ke <= 16 || (a.Ke % 64 == 0 && a.Ke <= 128));
  const bool fused_ega = eg_shape && a.infer;          // a3 + a4 + a5 + a6 (inference)
  const bool fused_eg = eg_shape && ctx->fuse_edge_gate && !fused_ega;
  if (fused_ega) {
    // e' (unless last), then g ⊙ h̄[s] summed per destination inside each 32-edge unit: g never
    // reaches HBM; segments crossing a unit boundary and nodes without in-edges are completed
    // by agg_fixup_kernel from the unit partials (fixed unit order)
    if (csr.E > 0 && (r = launch_edgegate<D>(ctx, csr, layer, a, st, partial)) < 0) return r;
    n += csr.E > 0 ? r : 0;
    if (csr.N > 0) {
      const int grid = int(std::min<long>((long(csr.N) + 255) / 256, 8L * ctx->num_sms));
      OCCU_PROF_BEGIN(ctx, "agg_fixup", st);
      agg_fixup_kernel<<<grid, 256, 0, st>>>(csr.in_ptr, csr.N, D, partial,
                                             ctx->cfg.aggr == OCCU_AGGR_MEAN, slope, a.h_out);
      OCCU_PROF_END(ctx);
      TC_CHECK();
      ++n;
    }
    return n;
  }
  if (csr.E > 0 && fused_eg) {
    // a3 + a4 fused: e' and g in one kernel (e' is not re-read)
    if ((r = launch_edgegate<D>(ctx, csr, layer, a, st)) < 0) return r;
    n += r;
  } else if (csr.E > 0) {
    // a3: edge transform
    if (a.Ke <= 16) {
      const int grid = int(std::min<long>((long(csr.E) + 255) / 256, 8L * ctx->num_sms));
      OCCU_PROF_BEGIN(ctx, "edge_small", st);
      if (a.Ke <= 4)
        launch_pdl(ctx->pdl & 4, edge_small_kernel<D, 4>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke, a.W_e,
                   a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, a.e_out, a.e0_out);
      else
        launch_pdl(ctx->pdl & 4, edge_small_kernel<D, 16>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke, a.W_e,
                   a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, a.e_out, a.e0_out);
      OCCU_PROF_END(ctx);
      TC_CHECK();
      ++n;
    } else {
      RowGemmArgs re{};
      re.slope = slope;
      re.A = a.e_in; re.K = a.Ke; re.R = csr.E; re.W = a.W_e; re.out = a.e_out;
      re.wimg = tc_wimg(ctx, 1, layer); re.wfexp = tc_wfexp(ctx, 1, layer);
      re.pin = a.p; re.qin = a.q; re.src = csr.in_src; re.dst = csr.in_dst;
      if ((r = launch_rowgemm<D, EPI_EDGE>(ctx, re, "edge_tc", st)) < 0) return r;
      n += r;
    }
    if (ctx->path == 2) {
      // a4 + a5 + a6 fused: channel-softmax gate, message, segmented sum, LeakyReLU
      RowGemmArgs rg{};
      rg.slope = slope;
      rg.A = a.e_out; rg.K = D; rg.R = csr.E; rg.W = a.W_m; rg.out = a.h_out;
      rg.wimg = tc_wimg(ctx, 2, layer); rg.wfexp = tc_wfexp(ctx, 2, layer);
      rg.hbar = a.hbar; rg.src = csr.in_src; rg.dst = csr.in_dst; rg.in_ptr = csr.in_ptr;
      rg.mean = ctx->cfg.aggr == OCCU_AGGR_MEAN; rg.part = partial;
      if ((r = launch_rowgemm<D, EPI_GATEAGG>(ctx, rg, "gate_agg_tc", st)) < 0) return r;
      n += r;
    } else if (ctx->cfg.msg == OCCU_MSG_NEIGHBOR_SOFTMAX) {
      // a4 under reading B: logits v = W_m e' -> g (the softmax runs in the aggregation)
      if ((r = launch_plain_tc(ctx, a.e_out, D, csr.E, 2, layer, nullptr, a.g, "gate_tc", st)) < 0)
        return r;
      n += r;
    } else {
      // a4: channel-softmax gate -> g
      RowGemmArgs rg{};
      rg.slope = slope;
      rg.A = a.e_out; rg.K = D; rg.R = csr.E; rg.W = a.W_m; rg.out = a.g;
      rg.wimg = tc_wimg(ctx, 2, layer); rg.wfexp = tc_wfexp(ctx, 2, layer);
      rg.rev = ctx->l2_order;
      if ((r = launch_rowgemm<D, EPI_GATE>(ctx, rg, "gate_tc", st)) < 0) return r;
      n += r;
    }
  }
  if (ctx->path == 2) {
    if (csr.N > 0) {
      const int grid = int(std::min<long>((long(csr.N) + 255) / 256, 8L * ctx->num_sms));
      OCCU_PROF_BEGIN(ctx, "agg_fixup", st);
      agg_fixup_kernel<<<grid, 256, 0, st>>>(csr.in_ptr, csr.N, D, partial,
                                             ctx->cfg.aggr == OCCU_AGGR_MEAN, slope, a.h_out);
      OCCU_PROF_END(ctx);
      TC_CHECK();
      ++n;
    }
  } else if (ctx->cfg.msg == OCCU_MSG_NEIGHBOR_SOFTMAX) {
    // a5 + a6 under reading B: segmented per-channel softmax + message + sum
    if ((r = launch_gather_segsoftmax(ctx, csr, a.g, a.hbar, a.h_out, a.rpart, a.save_w, st)) < 0)
      return r;
    n += r;
  } else {
    // a5 + a6: gather + segmented sum (CUDA cores, warp per 8 destinations)
    if ((r = launch_gather_segsum(ctx, csr, a.g, a.hbar, a.h_out, a.rpart, st, a.h_bits)) < 0) return r;
    n += r;
  }
  return n;
}

// ---- backward row-GEMMs on tensor cores ------------------------------------
template <int D>
static int bwd_gate_impl(const occu_ctx *ctx, const DevCsr &csr, int layer, const float *e,
                         const float *dh, const float *h, const float *hbar, float *MG, float *DV,
                         cudaStream_t st) {
  RowGemmArgs r{};
  r.slope = ctx->cfg.slope;
  r.A = e; r.K = D; r.R = csr.E; r.out = MG; r.out2 = DV;
  r.wimg = tc_wimg(ctx, 2, layer); r.wfexp = tc_wfexp(ctx, 2, layer);
  r.dh = dh; r.h = h; r.hbar = hbar; r.src = csr.in_src; r.dst = csr.in_dst;
  r.in_ptr = csr.in_ptr; r.mean = ctx->cfg.aggr == OCCU_AGGR_MEAN;
  return launch_rowgemm<D, EPI_GATEBWD>(ctx, r, "gate_bwd_tc", st);
}
template <int D>
static int plain_impl(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                      const float *add, float *out, const char *name, cudaStream_t st,
                      const float *mask_h, const int32_t *in_ptr, bool mask_bf, const uint32_t *mask_bits,
                      const int *rexp) {
  RowGemmArgs r{};
  r.mask_bf = mask_bf ? 1 : 0;
  r.mask_bits = mask_bits;
  r.rexp = rexp;
  r.slope = ctx->cfg.slope;
  r.A = A; r.K = K; r.R = R; r.add = add; r.out = out;
  r.wimg = tc_wimg(ctx, wkind, layer); r.wfexp = tc_wfexp(ctx, wkind, layer);
  r.mask_h = mask_h; r.in_ptr = in_ptr; r.mean = ctx->cfg.aggr == OCCU_AGGR_MEAN;
  return launch_rowgemm<D, EPI_PLAIN>(ctx, r, name, st);
}
template <int D>
static int plain_masked_impl(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                             const float *add, float *out, const char *name, cudaStream_t st,
                             const float *mask, float slope) {
  RowGemmArgs r{};
  r.slope = slope;
  r.A = A; r.K = K; r.R = R; r.add = add; r.out = out;
  r.wimg = tc_wimg(ctx, wkind, layer); r.wfexp = tc_wfexp(ctx, wkind, layer);
  r.mask_h = mask; r.mean = 0;
  return launch_rowgemm<D, EPI_PLAIN>(ctx, r, name, st);
}
int launch_plain_masked_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                           const float *add, float *out, const char *name, cudaStream_t st,
                           const float *mask, float slope) {
  if (R <= 0) return 0;
  return ctx->cfg.d == 64 ? plain_masked_impl<64>(ctx, A, K, R, wkind, layer, add, out, name, st, mask, slope)
                          : plain_masked_impl<128>(ctx, A, K, R, wkind, layer, add, out, name, st, mask, slope);
}
template <int D>
static int bias_impl(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                     const float *bias, bool relu, float *out, const char *name, cudaStream_t st) {
  RowGemmArgs r{};
  r.slope = ctx->cfg.slope;
  r.A = A; r.K = K; r.R = R; r.out = out; r.bias = bias; r.relu = relu ? 1 : 0;
  r.wimg = tc_wimg(ctx, wkind, layer); r.wfexp = tc_wfexp(ctx, wkind, layer);
  return launch_rowgemm<D, EPI_PLAIN>(ctx, r, name, st);
}
template <int D>
static int bwd_edge_impl(const occu_ctx *ctx, const DevCsr &csr, int layer, const float *e_in,
                         int Ke, const float *e, const float *de, const float *p, const float *q,
                         float *DZ, float *dal, cudaStream_t st, int *dz_rexp) {
  RowGemmArgs r{};
  r.out_rexp = dz_rexp;
  r.slope = ctx->cfg.slope;
  r.A = e_in; r.K = Ke; r.R = csr.E; r.out = DZ; r.dal = dal;
  r.wimg = tc_wimg(ctx, 1, layer); r.wfexp = tc_wfexp(ctx, 1, layer);
  // e' is recomputed in the epilogue (σ of the recomputed αz) when the forward formed it with
  // the same row-GEMM (EPI_EDGE); the fused edge+gate forward stores it from another kernel
  r.e = ctx->fuse_edge_gate ? e : nullptr;
  r.de = de; r.pin = p; r.qin = q; r.src = csr.in_src; r.dst = csr.in_dst;
  return launch_rowgemm<D, EPI_EDGEBWD>(ctx, r, "edge_bwd_tc", st);
}

int launch_bwd_gate_tc(const occu_ctx *ctx, const DevCsr &csr, int layer, const float *e,
                       const float *dh, const float *h, const float *hbar, float *MG, float *DV,
                       cudaStream_t st) {
  if (csr.E <= 0) return 0;
  return ctx->cfg.d == 64 ? bwd_gate_impl<64>(ctx, csr, layer, e, dh, h, hbar, MG, DV, st)
                          : bwd_gate_impl<128>(ctx, csr, layer, e, dh, h, hbar, MG, DV, st);
}
int launch_plain_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                    const float *add, float *out, const char *name, cudaStream_t st,
                    const float *mask_h, const int32_t *in_ptr, bool mask_bf, const uint32_t *mask_bits,
                    const int *rexp) {
  if (R <= 0) return 0;
  return ctx->cfg.d == 64 ? plain_impl<64>(ctx, A, K, R, wkind, layer, add, out, name, st, mask_h, in_ptr, mask_bf, mask_bits, rexp)
                          : plain_impl<128>(ctx, A, K, R, wkind, layer, add, out, name, st, mask_h, in_ptr, mask_bf, mask_bits, rexp);
}
int launch_bias_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                   const float *bias, bool relu, float *out, const char *name, cudaStream_t st) {
  if (R <= 0) return 0;
  return ctx->cfg.d == 64 ? bias_impl<64>(ctx, A, K, R, wkind, layer, bias, relu, out, name, st)
                          : bias_impl<128>(ctx, A, K, R, wkind, layer, bias, relu, out, name, st);
}
template <int D>
static int bias_add_impl(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                         const float *bias, const float *add, float *out, const char *name,
                         cudaStream_t st) {
  RowGemmArgs r{};
  r.slope = ctx->cfg.slope;
  r.A = A; r.K = K; r.R = R; r.out = out; r.bias = bias; r.add = add;
  r.wimg = tc_wimg(ctx, wkind, layer); r.wfexp = tc_wfexp(ctx, wkind, layer);
  return launch_rowgemm<D, EPI_PLAIN>(ctx, r, name, st);
}
// out = A·Wᵀ + bias + add (residual), rows R (Graphormer output projections)
int launch_bias_add_tc(const occu_ctx *ctx, const float *A, int K, int R, int wkind, int layer,
                       const float *bias, const float *add, float *out, const char *name,
                       cudaStream_t st) {
  if (R <= 0) return 0;
  return ctx->cfg.d == 64 ? bias_add_impl<64>(ctx, A, K, R, wkind, layer, bias, add, out, name, st)
                          : bias_add_impl<128>(ctx, A, K, R, wkind, layer, bias, add, out, name, st);
}
int launch_bwd_edge_tc(const occu_ctx *ctx, const DevCsr &csr, int layer, const float *e_in, int Ke,
                       const float *e, const float *de, const float *p, const float *q, float *DZ,
                       float *dal, cudaStream_t st, int *dz_rexp) {
  if (csr.E <= 0) return 0;
  return ctx->cfg.d == 64 ? bwd_edge_impl<64>(ctx, csr, layer, e_in, Ke, e, de, p, q, DZ, dal, st, dz_rexp)
                          : bwd_edge_impl<128>(ctx, csr, layer, e_in, Ke, e, de, p, q, DZ, dal, st, dz_rexp);
}

// OCCU_BF16 at d = 256 (kernels_bf16.cu): the pair row-GEMM of one forward step.
// epi: 0 node (A = layer-1 FP32 features if af32, else BF16 h), 1 edge, 2 gate; out BF16.
int launch_pair_bf16(const occu_ctx *ctx, int epi, bool af32, const void *A, int K, int R, int layer,
                     void *out, const float *a_s, const float *a_d, float *p, float *q,
                     const int32_t *src, const int32_t *dst, const char *name, cudaStream_t st) {
  RowGemmArgs ra{};
  ra.slope = ctx->cfg.slope;
  ra.A = static_cast<const float *>(A); ra.K = K; ra.R = R;
  ra.out = static_cast<float *>(out);
  ra.wimg = tc_wimg(ctx, epi, layer); ra.wfexp = tc_wfexp(ctx, epi, layer);
  ra.a_s = a_s; ra.a_d = a_d; ra.p = p; ra.q = q;
  ra.pin = p; ra.qin = q; ra.src = src; ra.dst = dst;
  ra.rev = epi == 1 ? 0 : ctx->l2_order;
  switch (epi * 2 + (af32 ? 1 : 0)) {
    case 0: return launch_rowgemm_pair<EPI_NODE, true, false>(ctx, ra, name, st);
    case 1: return launch_rowgemm_pair<EPI_NODE, true, true>(ctx, ra, name, st);
    case 2: return launch_rowgemm_pair<EPI_EDGE, true, false>(ctx, ra, name, st);
    case 3: return launch_rowgemm_pair<EPI_EDGE, true, true>(ctx, ra, name, st);
    case 4: return launch_rowgemm_pair<EPI_GATE, true, false>(ctx, ra, name, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

int launch_forward_layer_tc(const occu_ctx *ctx, const DevCsr &csr, int layer, const FwdLayerArgs &a,
                            float *partial, cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return tc_forward_layer_impl<64>(ctx, csr, layer, a, partial, st);
    case 128: return tc_forward_layer_impl<128>(ctx, csr, layer, a, partial, st);
    case 256:
      if (ctx->cfg.msg != OCCU_MSG_CHANNEL_SOFTMAX) return -int(cudaErrorInvalidValue);
      return tc_forward_layer_pair(ctx, csr, layer, a, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

}  // namespace occu

#ifdef OCCU_TC_TIMING
extern "C" int occu_debug_tc_time(unsigned long long *host) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(host, occu::g_tc_time, sizeof(occu::g_tc_time));
  static unsigned long long zero[32][4] = {};
  cudaMemcpyToSymbol(occu::g_tc_time, zero, sizeof(zero));
  return 0;
}
extern "C" int occu_debug_eg_time(unsigned long long *host) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(host, occu::g_eg_time, sizeof(occu::g_eg_time));
  static unsigned long long zero[32][4] = {};
  cudaMemcpyToSymbol(occu::g_eg_time, zero, sizeof(zero));
  return 0;
}
#endif

