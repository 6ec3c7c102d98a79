// OCCU_BF16 forward row-GEMMs on tcgen05 (SURVEY §8(c) "Precision modes", OCCU_BF16):
// GEMM operands are BF16 (the weights and the activations fed to the MMA: h, e, e'),
// the stored activations h̄, e' (and the gate scratch g, R24) are BF16, the
// MMAs accumulate in FP32 (TMEM), and p, q, α, σ, the softmax, the message product,
// the segmented sums, the readout and the head stay FP32.  Tolerance 1e-2 (north_star).
//
// rowgemm_bf16_kernel<D, EPI, AF32> computes, for 128-row tiles of an [R][K] input,
// acc = A·Wᵀ (one kind::f16 BF16 product per 16-wide K step) and a fused epilogue:
//   EPI_NODE : h̄ = LReLU(acc) -> BF16, p = h̄·a_s, q = h̄·a_d (FP32)        (a2, P141-P147)
//   EPI_EDGE : e' = σ(α·acc), α = p[s] + q[t] -> BF16                       (a3, P145)
//   EPI_GATE : g = softmax_c(acc) -> BF16                                   (a4, P149)
//   EPI_EDGEBWD (training, R28): z = acc recomputed exactly as the forward's EPI_EDGE;
//              dy = de ⊙ e' ⊙ σ(-αz) (BF16 e', FP32 de), dα = <dy, z> (float64), DZ = α dy
//              -> FP32                                                      (a10, SURVEY §8(c) BW)
// Input BF16 (layers >= 2): TMA writes the tile in the canonical SW128 K-major layout and
// the MMA reads it straight from shared memory (no conversion pass).  Input FP32 (the
// layer-1 node features): converter warps round it to BF16 into TMEM (".ts" form).
// Warp roles: 0 producer (weights bulk copy + TMA ring), 1 MMA issuer, 2-9 converters
// (AF32 only), 10-25 two epilogue groups of 8 warps (2 warps per row, D/2 columns each)
// on alternating tiles with double-buffered TMEM accumulators.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>

#include "occu_internal.h"
#include "tc_common.cuh"

namespace occu {
namespace {

constexpr int TM = 128;
constexpr int NTH = 832;
constexpr int EPI0 = 10;
constexpr int EPI_NODE = 0, EPI_EDGE = 1, EPI_GATE = 2, EPI_LOGIT = 3, EPI_EDGEBWD = 5;
constexpr float LOG2E = 1.4426950408889634f;

__device__ __forceinline__ float lrelu(float x, float s) { return x > 0.f ? x : s * x; }
__device__ __forceinline__ float ex2(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float fast_rcp(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  const __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<const uint32_t *>(&h);
}

struct BfArgs {
  int K, R;
  const uint8_t *wimg;       // BF16 SW128 K-major image of W ([Kpad/64][D][128 B])
  const int *wf;             // [f (= 0), softmax no-shift flag]
  __nv_bfloat16 *out;        // [R][D]
  const float *a_s, *a_d;    // NODE
  float *p, *q;              // NODE outputs
  const float *pin, *qin;    // EDGE
  const int32_t *src, *dst;  // EDGE, EDGEBWD
  const __nv_bfloat16 *eb;   // EDGEBWD: e' [R][D]
  const float *de;           // EDGEBWD: de [R][D]
  float *outf;               // EDGEBWD: DZ [R][D]
  float *dal;                // EDGEBWD: dα [R]
  float slope;
  int rev;
};

__host__ __device__ inline int kpad64(int K) { return (K + 63) / 64 * 64; }
// ring slot bytes: BF16 input = Kpad/64 boxes of 128 rows x 128 B; FP32 input = ceil(K/32)
// boxes of 128 rows x 32 fp32
__host__ __device__ inline int slot_bytes(int K, bool af32) {
  return af32 ? (K + 31) / 32 * 16384 : kpad64(K) / 64 * 16384;
}
__host__ __device__ inline int ring_slots(bool af32) { return af32 ? 2 : 4; }
constexpr int XB_WORDS = 32 * 12;   // per-warp transpose buffer: 32 rows x (8 + 4 pad) words
__host__ __device__ inline size_t bf_smem_bytes(int D, int K, bool af32) {
  return 1024 + size_t(kpad64(K)) * D * 2 + size_t(ring_slots(af32)) * slot_bytes(K, af32) + 512 +
         3 * 2 * 2 * 128 * 4 + 2 * D * 4 + 24 * XB_WORDS * 4;
}

// Coalesced BF16 store of a 16-column chunk of the warp's 32 rows (thread = row):
// each row's 32-byte segment is one full sector; two rows per 64-byte lane pair.
__device__ __forceinline__ void warp_store_bf16(uint32_t *buf, __nv_bfloat16 *__restrict__ out,
                                                long wrow0, int wrows, int c0, int D,
                                                const float (&v)[16], int lane) {
  uint32_t w[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) w[u] = pack_bf16(v[2 * u], v[2 * u + 1]);
  uint32_t *b = buf + lane * 12;
  *reinterpret_cast<uint4 *>(b) = make_uint4(w[0], w[1], w[2], w[3]);
  *reinterpret_cast<uint4 *>(b + 4) = make_uint4(w[4], w[5], w[6], w[7]);
  __syncwarp();
#pragma unroll
  for (int it = 0; it < 2; ++it) {
    const int idx = it * 32 + lane, r = idx >> 1, h = idx & 1;
    if (r < wrows)
      *reinterpret_cast<uint4 *>(out + (wrow0 + r) * D + c0 + h * 8) =
          *reinterpret_cast<const uint4 *>(buf + r * 12 + h * 4);
  }
  __syncwarp();
}

// Coalesced FP32 store of a 16-column chunk of the warp's 32 rows (thread = row), two
// 16-row passes through a 16 x 20 per-warp buffer (full 64-byte row segments).
__device__ __forceinline__ void warp_store_f32(float *buf, float *__restrict__ out, long wrow0,
                                               int wrows, int c0, int D, const float (&v)[16],
                                               int lane) {
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

__device__ __forceinline__ void group_bar(int g) {
  asm volatile("bar.sync %0, 256;" ::"r"(1 + g) : "memory");
}

template <int D, int EPI, bool AF32>
__global__ void __launch_bounds__(NTH, 1) rowgemm_bf16_kernel(const __grid_constant__ CUtensorMap tmap,
                                                              BfArgs a) {
  extern __shared__ uint8_t smem_raw[];
  const int K = a.K, Kp = kpad64(K), SB = slot_bytes(K, AF32), NS = ring_slots(AF32);
  uint8_t *base = smem_raw + ((1024 - (tc::smem_u32(smem_raw) & 1023)) & 1023);
  uint8_t *wimg = base;
  uint8_t *ring = base + size_t(Kp) * D * 2;
  uint8_t *misc = ring + size_t(NS) * SB;
  uint64_t *bars = reinterpret_cast<uint64_t *>(misc);
  uint64_t *full = bars, *empty = bars + 4, *afull = bars + 8, *afree = bars + 10,
           *accfull = bars + 12, *accfree = bars + 15, *wfull = bars + 18;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(misc + 256);
  float *xch = reinterpret_cast<float *>(misc + 512);              // [3 groups][2][2][128]
  float *avec = xch + 3 * 2 * 2 * 128;                             // [2*D]
  uint32_t *xbuf = reinterpret_cast<uint32_t *>(avec + 2 * D);     // 24 x XB_WORDS
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  pdl_trigger();
  if (threadIdx.x == 0) {
    for (int j = 0; j < 4; ++j) {
      tc::mbar_init(full + j, 1);
      tc::mbar_init(empty + j, AF32 ? 256 : 1);
    }
    for (int j = 0; j < 2; ++j) {
      tc::mbar_init(afull + j, 256);
      tc::mbar_init(afree + j, 1);
    }
    for (int j = 0; j < 3; ++j) {
      tc::mbar_init(accfull + j, 1);
      tc::mbar_init(accfree + j, 256);
    }
    tc::mbar_init(wfull, 1);
    tc::fence_mbar_init();
  }
  if (warp == 1) tc::tmem_alloc<512>(tmem_slot);
  pdl_wait();                              // predecessor's writes visible from here on
  if (EPI == EPI_NODE)
    for (int i = threadIdx.x; i < D; i += NTH) {
      avec[i] = a.a_s[i];
      avec[D + i] = a.a_d[i];
    }
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  const uint32_t tmem = *tmem_slot;
  const int tiles = (a.R + TM - 1) / TM;
  const int my = blockIdx.x < tiles ? (tiles - 1 - int(blockIdx.x)) / int(gridDim.x) + 1 : 0;
  auto tile_r0 = [&](int i) -> long {
    const int t = int(blockIdx.x) + i * int(gridDim.x);
    return long(a.rev ? tiles - 1 - t : t) * TM;
  };
  auto a_col = [](int j) { return uint32_t(j) * 128u; };
  // BF16 input: no TMEM A operand and no converters, so the converter warps form a third
  // epilogue group and three accumulators rotate (cols 0/128/256); FP32 input: A[2] at
  // cols 0/128, two accumulators at 256/384, two epilogue groups.
  constexpr int NG = AF32 ? 2 : 3;
  constexpr int EW0 = AF32 ? EPI0 : 2;
  auto acc_col = [](int j) { return (AF32 ? 256u : 0u) + uint32_t(j) * 128u; };

  if (warp == 0) {
    if (lane == 0) {
      tc::prefetch_tmap(&tmap);
      const uint32_t ib = uint32_t(Kp) * D * 2;
      tc::mbar_arrive_expect_tx(wfull, ib);
      for (uint32_t o = 0; o < ib; o += 16384) tc::bulk_g2s(wimg + o, a.wimg + o, min(16384u, ib - o), wfull);
      const int nbox = SB / 16384;
      for (int i = 0; i < my; ++i) {
        const int s = i % NS;
        if (i >= NS) tc::mbar_wait(empty + s, ((i / NS) - 1) & 1);
        tc::mbar_arrive_expect_tx(full + s, uint32_t(SB));
        const int r0 = int(tile_r0(i));
        for (int b = 0; b < nbox; ++b)
          tc::tma_load_2d(ring + size_t(s) * SB + b * 16384, &tmap, (AF32 ? 32 : 64) * b, r0, full + s);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    const uint32_t idsc = tc::idesc(128, uint32_t(D), tc::FMT_BF16);
    const uint32_t wa = tc::smem_u32(wimg);
    const uint32_t ra = tc::smem_u32(ring);
    const int nk = Kp / 16;
    tc::mbar_wait(wfull, 0);
    for (int i = 0; i < my; ++i) {
      const int j = i & 1, s = i % NS, ja = i % NG;
      if (AF32) tc::mbar_wait(afull + j, (i >> 1) & 1);
      else tc::mbar_wait(full + s, (i / NS) & 1);
      if (i >= NG) tc::mbar_wait(accfree + ja, ((i / NG) - 1) & 1);
      tc::fence_after_sync();
      if (lane == 0) {
        const uint32_t d = tmem + acc_col(ja);
        for (int kk = 0; kk < nk; ++kk) {
          const uint32_t boff = uint32_t(kk >> 2) * uint32_t(D) * 128u + uint32_t(kk & 3) * 32u;
          const uint64_t bdesc = tc::sdesc_sw128(wa + boff);
          if (AF32) {
            tc::mma_f16_ts(d, tmem + a_col(j) + uint32_t(kk) * 8u, bdesc, idsc, kk > 0 ? 1u : 0u);
          } else {
            const uint32_t aoff = uint32_t(s) * SB + uint32_t(kk >> 2) * 16384u + uint32_t(kk & 3) * 32u;
            tc::mma_f16_ss(d, tc::sdesc_sw128(ra + aoff), bdesc, idsc, kk > 0 ? 1u : 0u);
          }
        }
        tc::mma_commit(accfull + ja);
        if (AF32) tc::mma_commit(afree + j);
        else tc::mma_commit(empty + s);
      }
      __syncwarp();
    }
  } else if (warp < EW0) {
    {
      // converters: thread = (row, K-half), FP32 -> BF16 pairs -> TMEM A[j]
      const int qd = warp & 3, kh = (warp - 2) >> 2, row = qd * 32 + lane;
      const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
      const int KH = Kp / 2, kb = kh * KH;
      for (int i = 0; i < my; ++i) {
        const int j = i & 1, s = i % NS;
        const long r0 = tile_r0(i);
        const bool live = row < min(TM, int(a.R - r0));
        tc::mbar_wait(full + s, (i / NS) & 1);
        if (i >= 2) tc::mbar_wait(afree + j, ((i >> 1) - 1) & 1);
        const float *sl = reinterpret_cast<const float *>(ring + size_t(s) * SB);
        for (int c0 = 0; c0 < KH / 2; c0 += 16) {
          uint32_t x[16];
#pragma unroll
          for (int u = 0; u < 16; u += 2) {
            const int k = kb + 2 * (c0 + u);
            float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
            if (live && k < K) {
              const int b = k >> 5, c = (k & 31) >> 2;
              v = *reinterpret_cast<const float4 *>(sl + b * 4096 + row * 32 + ((c ^ (row & 7)) << 2));
            }
            x[u] = pack_bf16(v.x, v.y);
            x[u + 1] = pack_bf16(v.z, v.w);
          }
          tc::tmem_st16(lane_base + a_col(j) + uint32_t(kb / 2 + c0), x);
        }
        tc::tmem_st_wait();
        tc::fence_before_sync();
        tc::mbar_arrive(empty + s);
        tc::mbar_arrive(afull + j);
      }
    }
  } else {
    // ---------------- epilogue: two groups of 8 warps on alternating tiles ----------------
    const int wi = warp - EW0, g = wi >> 3, hf = (wi >> 2) & 1, qd = warp & 3;
    const int row = qd * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t(qd * 32) << 16);
    float *xg = xch + g * (2 * 2 * 128);
    uint32_t *wbuf = xbuf + wi * XB_WORDS;
    constexpr int DH = D / 2;
    const int cb = hf * DH;
    const bool noshift = EPI == EPI_GATE && __ldg(a.wf + 1) != 0;
    for (int i = g; i < my; i += NG) {
      const int j = i % NG;
      const long r0 = tile_r0(i);
      const int nrows = min(TM, int(a.R - r0));
      const bool live = row < nrows;
      const long grow = r0 + row;
      const long wrow0 = r0 + qd * 32;
      const int wrows = max(0, min(32, nrows - qd * 32));
      float al = 0.f;
      if ((EPI == EPI_EDGE || EPI == EPI_EDGEBWD) && live)
        al = __ldg(a.pin + __ldg(a.src + grow)) + __ldg(a.qin + __ldg(a.dst + grow));
      tc::mbar_wait(accfull + j, (i / NG) & 1);
      tc::fence_after_sync();
      const uint32_t acc = lane_base + acc_col(j) + cb;
      if (EPI == EPI_NODE) {
        float pp = 0.f, qq = 0.f;
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) {
            o[u] = lrelu(__uint_as_float(r[u]), a.slope);
            pp = fmaf(o[u], avec[cb + c0 + u], pp);
            qq = fmaf(o[u], avec[D + cb + c0 + u], qq);
          }
          warp_store_bf16(wbuf, a.out, wrow0, wrows, cb + c0, D, o, lane);
        }
        xg[hf * 128 + row] = pp;
        xg[256 + hf * 128 + row] = qq;
        group_bar(g);
        if (hf == 0 && live) {
          a.p[grow] = pp + xg[128 + row];
          a.q[grow] = qq + xg[256 + 128 + row];
        }
      } else if (EPI == EPI_EDGE) {
        const float cexp = -al * LOG2E;
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = fast_rcp(1.f + ex2(__uint_as_float(r[u]) * cexp));  // e' (R2, R3)
          warp_store_bf16(wbuf, a.out, wrow0, wrows, cb + c0, D, o, lane);
        }
      } else if (EPI == EPI_LOGIT) {      // reading B: the logits v = W_m e' -> BF16
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) o[u] = __uint_as_float(r[u]);
          warp_store_bf16(wbuf, a.out, wrow0, wrows, cb + c0, D, o, lane);
        }
      } else if (EPI == EPI_EDGEBWD) {
        const float cexp = al * LOG2E;
        double dpart = 0.0;                       // dα = <dy, z> in float64 (cancellation)
#pragma unroll 1
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          float ev[16], dv[16];
          if (live) {
            const uint4 *ep = reinterpret_cast<const uint4 *>(a.eb + grow * D + cb + c0);
            const float4 *dp = reinterpret_cast<const float4 *>(a.de + grow * D + cb + c0);
            const uint4 e0 = __ldg(ep), e1 = __ldg(ep + 1);
            const uint32_t ew[8] = {e0.x, e0.y, e0.z, e0.w, e1.x, e1.y, e1.z, e1.w};
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              ev[2 * u] = __uint_as_float(ew[u] << 16);
              ev[2 * u + 1] = __uint_as_float(ew[u] & 0xFFFF0000u);
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              const float4 x = __ldg(dp + u);
              dv[4 * u] = x.x; dv[4 * u + 1] = x.y; dv[4 * u + 2] = x.z; dv[4 * u + 3] = x.w;
            }
          } else {
#pragma unroll
            for (int u = 0; u < 16; ++u) ev[u] = dv[u] = 0.f;
          }
          tc::tmem_ld_wait();
          float o[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) {
            const float z = __uint_as_float(r[u]);
            // σ'(y) = σ(y)·σ(-y): σ(y) is the stored e', σ(-y) from the recomputed y = α z
            const float dy = dv[u] * ev[u] * fast_rcp(1.f + ex2(z * cexp));
            dpart = fma(double(dy), double(z), dpart);
            o[u] = al * dy;
          }
          warp_store_f32(reinterpret_cast<float *>(wbuf), a.outf, wrow0, wrows, cb + c0, D, o, lane);
        }
        double *xd = reinterpret_cast<double *>(xg);   // the group's exchange area
        xd[hf * 128 + row] = dpart;
        group_bar(g);
        if (hf == 0 && live) a.dal[grow] = float(dpart + xd[128 + row]);
      } else {
        float m = 0.f;
        if (!noshift) {
          m = -INFINITY;
#pragma unroll
          for (int c0 = 0; c0 < DH; c0 += 16) {
            uint32_t r[16];
            tc::tmem_ld16(acc + c0, r);
            tc::tmem_ld_wait();
#pragma unroll
            for (int u = 0; u < 16; ++u) m = fmaxf(m, __uint_as_float(r[u]));
          }
          xg[hf * 128 + row] = m;
          group_bar(g);
          m = fmaxf(m, xg[(hf ^ 1) * 128 + row]);
        }
        const float mL = m * LOG2E;
        float sum = 0.f;
#pragma unroll
        for (int c0 = 0; c0 < DH; c0 += 16) {
          uint32_t r[16];
          tc::tmem_ld16(acc + c0, r);
          tc::tmem_ld_wait();
#pragma unroll
          for (int u = 0; u < 16; ++u) sum += ex2(fmaf(__uint_as_float(r[u]), LOG2E, -mL));
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
          for (int u = 0; u < 16; ++u) o[u] = ex2(fmaf(__uint_as_float(r[u]), LOG2E, -mL)) * inv;
          warp_store_bf16(wbuf, a.out, wrow0, wrows, cb + c0, D, o, lane);
        }
      }
      tc::fence_before_sync();
      tc::mbar_arrive(accfree + j);
      group_bar(g);          // the exchange slots are reused by the next tile
    }
  }
  tc::fence_before_sync();
  __syncthreads();
  tc::fence_after_sync();
  if (warp == 1) tc::tmem_dealloc<512>(tmem);
}

// Layer-1 edge transform in BF16 mode: as edge_small_kernel (FP32 math on CUDA cores, the
// a1 permutation fused through in_eid), storing e' as BF16.
template <int D, int KM>
__global__ void __launch_bounds__(256) edge_small_bf16_kernel(
    const float *__restrict__ e_in, int Ke, const float *__restrict__ W_e,
    const float *__restrict__ p, const float *__restrict__ q, const int32_t *__restrict__ in_src,
    const int32_t *__restrict__ in_dst, const int32_t *__restrict__ eid, int E,
    __nv_bfloat16 *__restrict__ e_out, float *__restrict__ e0_out) {
  constexpr int V = D / 32;
  extern __shared__ float wsm[];
  pdl_trigger();
  pdl_wait();
  for (int i = threadIdx.x; i < D * Ke; i += blockDim.x) wsm[(i % Ke) * D + i / Ke] = W_e[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int c = lane * V;
  float w[KM][V];
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
      const long rw = eid ? long(__ldg(eid + k)) : k;
#pragma unroll
      for (int j = 0; j < KM; ++j) ev[j] = j < Ke ? __ldg(e_in + rw * Ke + j) : 0.f;
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
      uint32_t o[V / 2];
#pragma unroll
      for (int v = 0; v < V; v += 2)
        o[v / 2] = pack_bf16(fast_rcp(1.f + ex2(-(a * z[v]) * LOG2E)),
                             fast_rcp(1.f + ex2(-(a * z[v + 1]) * LOG2E)));
      __nv_bfloat16 *dst = e_out + (k0 + u) * D + c;
      if constexpr (V == 8) *reinterpret_cast<uint4 *>(dst) = make_uint4(o[0], o[1 % (V / 2)], o[2 % (V / 2)], o[3 % (V / 2)]);
      else if constexpr (V == 4) *reinterpret_cast<uint2 *>(dst) = make_uint2(o[0], o[1 % (V / 2)]);
      else *reinterpret_cast<uint32_t *>(dst) = o[0];
    }
  }
}

using PFN_encodeTiled = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                     const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                     const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                     CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

bool encode_map(CUtensorMap *m, const void *A, int R, int K, bool bf16) {
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
  const cuuint64_t strides[1] = {cuuint64_t(K) * (bf16 ? 2 : 4)};
  const cuuint32_t box[2] = {bf16 ? 64u : 32u, 128u};
  const cuuint32_t estr[2] = {1, 1};
  return fn(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
            const_cast<void *>(A), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <class Kern> void set_smem(Kern k, size_t bytes) {
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes));
}

template <int D, int EPI, bool AF32>
int launch_bf(const occu_ctx *ctx, const BfArgs &ra, const void *A, const char *name, cudaStream_t st) {
  if (ra.R <= 0) return 0;
  const size_t smem = bf_smem_bytes(D, ra.K, AF32);
  set_smem(rowgemm_bf16_kernel<D, EPI, AF32>, smem);
  const int tiles = (ra.R + TM - 1) / TM;
  const int grid = std::min(tiles, ctx->num_sms);
  CUtensorMap tmap;
  if (!encode_map(&tmap, A, ra.R, ra.K, !AF32)) return -int(cudaErrorInvalidValue);
  OCCU_PROF_BEGIN(ctx, name, st);
  launch_pdl(ctx->pdl & 16, rowgemm_bf16_kernel<D, EPI, AF32>, grid, NTH, smem, st, tmap, ra);
  OCCU_PROF_END(ctx);
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 1 : -int(e);
}

template <int D>
int forward_layer_bf16(const occu_ctx *ctx, const DevCsr &csr, int layer, const FwdLayerArgs &a,
                       cudaStream_t st) {
  int n = 0, r;
  const float slope = ctx->cfg.slope;
  BfArgs ra{};
  ra.slope = slope;
  ra.rev = ctx->l2_order;
  // a2: node transform; layer 1 reads the FP32 node features, later layers BF16 h
  ra.K = a.K; ra.R = csr.N; ra.out = reinterpret_cast<__nv_bfloat16 *>(a.hbar);
  ra.wimg = tc_wimg(ctx, 0, layer); ra.wf = tc_wfexp(ctx, 0, layer);
  ra.a_s = a.a_s; ra.a_d = a.a_d; ra.p = a.p; ra.q = a.q;
  r = layer == 0 ? launch_bf<D, EPI_NODE, true>(ctx, ra, a.h_in, "node_tc", st)
                 : launch_bf<D, EPI_NODE, false>(ctx, ra, a.h_in, "node_tc", st);
  if (r < 0) return r;
  n += r;
  if (csr.E > 0) {
    __nv_bfloat16 *e_out = reinterpret_cast<__nv_bfloat16 *>(a.e_out);
    if (a.Ke <= 16) {
      const int grid = int(std::min<long>((long(csr.E) + 255) / 256, 8L * ctx->num_sms));
      OCCU_PROF_BEGIN(ctx, "edge_small", st);
      if (a.Ke <= 4)
        launch_pdl(ctx->pdl & 4, edge_small_bf16_kernel<D, 4>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke,
                   a.W_e, a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, e_out, a.e0_out);
      else
        launch_pdl(ctx->pdl & 4, edge_small_bf16_kernel<D, 16>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke,
                   a.W_e, a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, e_out, a.e0_out);
      OCCU_PROF_END(ctx);
      const cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return -int(e);
      ++n;
    } else {
      BfArgs re{};
      re.slope = slope;
      re.rev = 0;
      re.K = a.Ke; re.R = csr.E; re.out = e_out;
      re.wimg = tc_wimg(ctx, 1, layer); re.wf = tc_wfexp(ctx, 1, layer);
      re.pin = a.p; re.qin = a.q; re.src = csr.in_src; re.dst = csr.in_dst;
      // layer 1 with wide edge features reads the permuted FP32 e0; later layers BF16 e'
      r = layer == 0 ? launch_bf<D, EPI_EDGE, true>(ctx, re, a.e_in, "edge_tc", st)
                     : launch_bf<D, EPI_EDGE, false>(ctx, re, a.e_in, "edge_tc", st);
      if (r < 0) return r;
      n += r;
    }
    BfArgs rg{};
    rg.slope = slope;
    rg.rev = ctx->l2_order;
    rg.K = D; rg.R = csr.E; rg.out = reinterpret_cast<__nv_bfloat16 *>(a.g);
    rg.wimg = tc_wimg(ctx, 2, layer); rg.wf = tc_wfexp(ctx, 2, layer);
    if (ctx->cfg.msg == OCCU_MSG_NEIGHBOR_SOFTMAX) {       // reading B: logits, then the
      if ((r = launch_bf<D, EPI_LOGIT, false>(ctx, rg, a.e_out, "gate_tc", st)) < 0) return r;
    } else if ((r = launch_bf<D, EPI_GATE, false>(ctx, rg, a.e_out, "gate_tc", st)) < 0) {
      return r;
    }
    n += r;
  }
  if (ctx->cfg.msg == OCCU_MSG_NEIGHBOR_SOFTMAX) {          // segmented softmax over in-edges
    if ((r = launch_gather_segsoftmax_bf16(ctx, csr, a.g, a.hbar, a.h_out, a.rpart, a.save_w, st)) < 0) return r;
    return n + r;
  }
  if ((r = launch_gather_segsum_bf16(ctx, csr, a.g, a.hbar, a.h_out, a.rpart, st, a.h_bits)) < 0) return r;
  return n + r;
}

template <int D>
int bwd_edge_bf16(const occu_ctx *ctx, const DevCsr &csr, int layer, const void *e_in, int Ke,
                  const void *e, const float *de, const float *p, const float *q, float *DZ,
                  float *dal, cudaStream_t st) {
  BfArgs re{};
  re.slope = ctx->cfg.slope;
  re.rev = 0;
  re.K = Ke; re.R = csr.E;
  re.wimg = tc_wimg(ctx, 1, layer); re.wf = tc_wfexp(ctx, 1, layer);
  re.pin = p; re.qin = q; re.src = csr.in_src; re.dst = csr.in_dst;
  re.eb = reinterpret_cast<const __nv_bfloat16 *>(e);
  re.de = de; re.outf = DZ; re.dal = dal;
  return launch_bf<D, EPI_EDGEBWD, false>(ctx, re, e_in, "edge_bwd_tc", st);
}

}  // namespace

int launch_bwd_edge_bf16(const occu_ctx *ctx, const DevCsr &csr, int layer, const void *e_in,
                         int Ke, const void *e, const float *de, const float *p, const float *q,
                         float *DZ, float *dal, cudaStream_t st) {
  if (csr.E <= 0) return 0;
  if (Ke != ctx->cfg.d) return -int(cudaErrorInvalidValue);
  switch (ctx->cfg.d) {
    case 64: return bwd_edge_bf16<64>(ctx, csr, layer, e_in, Ke, e, de, p, q, DZ, dal, st);
    case 128: return bwd_edge_bf16<128>(ctx, csr, layer, e_in, Ke, e, de, p, q, DZ, dal, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

// d = 256 in OCCU_BF16: the three row-GEMMs on CTA pairs (launch_pair_bf16, kernels_tc.cu),
// the layer-1 edge transform and the aggregation as at d <= 128
static int forward_layer_bf16_256(const occu_ctx *ctx, const DevCsr &csr, int layer, const FwdLayerArgs &a,
                                  cudaStream_t st) {
  constexpr int D = 256;
  if (ctx->cfg.msg != OCCU_MSG_CHANNEL_SOFTMAX) return -int(cudaErrorInvalidValue);
  int n = 0, r;
  if ((r = launch_pair_bf16(ctx, 0, layer == 0, a.h_in, a.K, csr.N, layer, a.hbar, a.a_s, a.a_d, a.p, a.q,
                            nullptr, nullptr, "node_tc", st)) < 0) return r;
  n += r;
  if (csr.E > 0) {
    __nv_bfloat16 *e_out = reinterpret_cast<__nv_bfloat16 *>(a.e_out);
    if (a.Ke <= 16) {
      const int grid = int(std::min<long>((long(csr.E) + 255) / 256, 8L * ctx->num_sms));
      OCCU_PROF_BEGIN(ctx, "edge_small", st);
      if (a.Ke <= 4)
        launch_pdl(ctx->pdl & 4, edge_small_bf16_kernel<D, 4>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke,
                   a.W_e, a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, e_out, a.e0_out);
      else
        launch_pdl(ctx->pdl & 4, edge_small_bf16_kernel<D, 16>, grid, 256, D * a.Ke * 4, st, a.e_in, a.Ke,
                   a.W_e, a.p, a.q, csr.in_src, csr.in_dst, a.e_eid, csr.E, e_out, a.e0_out);
      OCCU_PROF_END(ctx);
      const cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return -int(e);
      ++n;
    } else {
      if ((r = launch_pair_bf16(ctx, 1, layer == 0, a.e_in, a.Ke, csr.E, layer, e_out, nullptr, nullptr,
                                a.p, a.q, csr.in_src, csr.in_dst, "edge_tc", st)) < 0) return r;
      n += r;
    }
    if ((r = launch_pair_bf16(ctx, 2, false, a.e_out, D, csr.E, layer, a.g, nullptr, nullptr, nullptr,
                              nullptr, nullptr, nullptr, "gate_tc", st)) < 0) return r;
    n += r;
  }
  if ((r = launch_gather_segsum_bf16(ctx, csr, a.g, a.hbar, a.h_out, a.rpart, st, a.h_bits)) < 0) return r;
  return n + r;
}

int launch_forward_layer_bf16(const occu_ctx *ctx, const DevCsr &csr, int layer,
                              const FwdLayerArgs &a, cudaStream_t st) {
  switch (ctx->cfg.d) {
    case 64: return forward_layer_bf16<64>(ctx, csr, layer, a, st);
    case 128: return forward_layer_bf16<128>(ctx, csr, layer, a, st);
    case 256: return forward_layer_bf16_256(ctx, csr, layer, a, st);
    default: return -int(cudaErrorInvalidValue);
  }
}

namespace {
// exact BF16 -> FP32 widening, 8 elements per thread (16-byte loads)
__global__ void __launch_bounds__(256) bf16_to_f32_kernel(const uint4 *__restrict__ src, size_t n8,
                                                          float4 *__restrict__ dst) {
  for (size_t i = blockIdx.x * size_t(256) + threadIdx.x; i < n8; i += size_t(gridDim.x) * 256) {
    const uint4 v = __ldg(src + i);
    dst[2 * i] = make_float4(__uint_as_float(v.x << 16), __uint_as_float(v.x & 0xFFFF0000u),
                             __uint_as_float(v.y << 16), __uint_as_float(v.y & 0xFFFF0000u));
    dst[2 * i + 1] = make_float4(__uint_as_float(v.z << 16), __uint_as_float(v.z & 0xFFFF0000u),
                                 __uint_as_float(v.w << 16), __uint_as_float(v.w & 0xFFFF0000u));
  }
}
}  // namespace

int launch_bf16_to_f32(const occu_ctx *ctx, const void *src, size_t n, float *dst, cudaStream_t st) {
  if (n % 8) return -int(cudaErrorInvalidValue);          // n = N·d, d in {64, 128}
  const size_t n8 = n / 8;
  const int grid = int(std::min<size_t>((n8 + 255) / 256, size_t(8) * ctx->num_sms));
  if (n8 == 0) return 0;
  OCCU_PROF_BEGIN(ctx, "bf16_to_f32", st);
  bf16_to_f32_kernel<<<grid, 256, 0, st>>>(static_cast<const uint4 *>(src), n8, reinterpret_cast<float4 *>(dst));
  OCCU_PROF_END(ctx);
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 1 : -int(e);
}

}  // namespace occu
