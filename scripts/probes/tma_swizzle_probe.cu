// Probe: where does TMA SWIZZLE_128B_ATOM_32B put element (row, col) of a 32 x 32 fp32 box?
// Prints, per row, the logical 32-byte chunk found at each physical 32-byte position.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
__global__ void k(const __grid_constant__ CUtensorMap m, float *out) {
  __shared__ __align__(1024) float s[32 * 32];
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)), "r"(4096));
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"((uint32_t)__cvta_generic_to_shared(s)), "l"((uint64_t)&m), "r"(0), "r"(0),
                 "r"((uint32_t)__cvta_generic_to_shared(&bar)) : "memory");
  }
  asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W;\n}" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) out[i] = s[i];
}
int main() {
  float h[32 * 32];
  for (int i = 0; i < 1024; ++i) h[i] = float(i);
  float *d, *o;
  cudaMalloc(&d, 4096); cudaMalloc(&o, 4096);
  cudaMemcpy(d, h, 4096, cudaMemcpyHostToDevice);
  typedef CUresult (*F)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *,
                        const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  void *p; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  for (int sw : {3, 4}) {
    CUtensorMap m;
    cuuint64_t dims[2] = {32, 32}, str[1] = {128};
    cuuint32_t box[2] = {32, 32}, es[2] = {1, 1};
    CUresult r = ((F)p)(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        (CUtensorMapSwizzle)sw, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    k<<<1, 128>>>(m, o);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(h, o, 4096, cudaMemcpyDeviceToHost);
    printf("swizzle %d (encode %d, run %s): row: logical 16B chunk at each physical 16B slot\n", sw, (int)r, cudaGetErrorString(e));
    for (int row = 0; row < 12; ++row) {
      printf("  row %2d:", row);
      for (int c = 0; c < 8; ++c) {
        int v = (int)h[row * 32 + c * 4];
        printf(" %d%s", (v % 32) / 4, (v / 32 != row) ? "!" : "");
      }
      printf("\n");
    }
  }
  return 0;
}
