// Micro-probe (sm_100a): shared-memory wavefront cost of 128-bit loads by address pattern, and
// mma.sync m16n8k8 TF32 throughput of one SM — sizing data for the CFG1 single-CTA GEMMs.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void lds_probe(int mode, int iters, float *out, long long *cyc) {
  __shared__ __align__(16) float s[8192];
  for (int i = threadIdx.x; i < 8192; i += blockDim.x) s[i] = i * 1e-3f;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  int addr;
  if (mode == 0) addr = 0;                         // all lanes one 16-byte word
  else if (mode == 1) addr = lane * 4;             // 32 distinct, conflict-free
  else if (mode == 2) addr = (lane >> 4) * 68;     // two addresses (two rows)
  else if (mode == 3) addr = (lane & 15) * 68;     // 16 distinct (rows of stride 68), duplicated
  else addr = lane * 68;                           // 32 distinct rows of stride 68
  float4 acc = make_float4(0, 0, 0, 0);
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const int a = (addr + (it & 7) * 512) & 8191;
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                 : "r"(static_cast<unsigned>(__cvta_generic_to_shared(s + a))));
    acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
  out[threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}
__global__ void mma_probe(int iters, float *out, long long *cyc) {
  const int lane = threadIdx.x & 31;
  unsigned a0 = __float_as_uint(lane * 1e-3f), a1 = a0 ^ 1, a2 = a0 ^ 2, a3 = a0 ^ 3, b0 = a0 ^ 4, b1 = a0 ^ 5;
  float c[4][4] = {};
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int q = 0; q < 4; ++q)
      asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                   : "+f"(c[q][0]), "+f"(c[q][1]), "+f"(c[q][2]), "+f"(c[q][3])
                   : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
  float s = 0;
  for (int q = 0; q < 4; ++q) s += c[q][0] + c[q][1] + c[q][2] + c[q][3];
  out[threadIdx.x] = s;
}
int main() {
  float *out; long long *cyc, h;
  cudaMalloc(&out, 4096 * 4); cudaMalloc(&cyc, 8);
  const int iters = 4096;
  const char *names[5] = {"one address", "32 distinct", "two rows", "16 distinct x2", "32 rows str68"};
  for (int mode = 0; mode < 5; ++mode)
    for (int nt : {32, 1024}) {
      lds_probe<<<1, nt>>>(mode, iters, out, cyc);
      cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
      printf("LDS.128 %-15s threads %4d: %.2f cycles per warp-instruction (SM)\n", names[mode], nt,
             double(h) / iters / (nt / 32));
    }
  for (int nt : {32, 128, 512, 1024}) {
    mma_probe<<<1, nt>>>(iters, out, cyc);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    const double macs = double(iters) * 4 * 16 * 8 * 8 * (nt / 32);
    printf("mma.sync m16n8k8 tf32, %4d threads: %.1f MAC/cycle/SM\n", nt, macs / double(h));
  }
  return 0;
}
