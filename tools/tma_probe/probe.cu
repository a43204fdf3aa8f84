// Minimal TMA probe: load one 4-D fp64 box into smem and copy it out.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>

__device__ __forceinline__ uint32_t s32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int VARIANT>
__global__ void probe(const __grid_constant__ CUtensorMap tmap, double* out, int n, int c0, int c1) {
  extern __shared__ __align__(128) unsigned char sm[];
  double* buf = (double*)sm;
  uint64_t* bar = (uint64_t*)(sm + 65536);
  if (threadIdx.x == 0) {
    if (VARIANT == 1) asm volatile("prefetch.tensormap [%0];" :: "l"((uint64_t)&tmap) : "memory");
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(s32(bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(s32(bar)), "r"(n * 8) : "memory");
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
      :: "r"(s32(buf)), "l"((uint64_t)&tmap), "r"(c0), "r"(c1), "r"(0), "r"(0), "r"(s32(bar)) : "memory");
  }
  uint32_t done = 0;
  do {
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(s32(bar)), "r"(0) : "memory");
  } while (!done);
  for (int t = threadIdx.x; t < n; t += blockDim.x) out[t] = buf[t];
}

extern "C" int probe_main(int variant) {
  int nx = 12, ny = 12, nz = 12, sy = 16;
  size_t sm_ = (size_t)sy * ny, sk = 5 * sm_;
  std::vector<double> h(sk * nz);
  for (size_t t = 0; t < h.size(); ++t) h[t] = (double)t;
  double *d, *o;
  cudaMalloc(&d, h.size() * 8); cudaMalloc(&o, 1 << 20);
  cudaMemcpy(d, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
  void* fn = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  CUtensorMap map;
  int UX = 36, UY = 14;
  cuuint64_t gdim[4] = {(cuuint64_t)nx, (cuuint64_t)ny, 5, (cuuint64_t)nz};
  cuuint64_t gstr[3] = {(cuuint64_t)sy * 8, sm_ * 8, sk * 8};
  cuuint32_t box[4] = {(cuuint32_t)UX, (cuuint32_t)UY, 5, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  if (variant == 2) { box[0] = 16; box[1] = 8; }
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, d, gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("variant %d encode=%d\n", variant, (int)r);
  int n = box[0] * box[1] * 5;
  cudaFuncSetAttribute(probe<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
  cudaFuncSetAttribute(probe<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
  if (variant == 1) probe<1><<<1, 128, 70000>>>(map, o, n, -2, -2);
  else probe<0><<<1, 128, 70000>>>(map, o, n, variant == 3 ? 0 : -2, variant == 3 ? 0 : -2);
  cudaError_t e = cudaDeviceSynchronize();
  printf("variant %d: %s\n", variant, cudaGetErrorString(e));
  std::vector<double> ho(n);
  cudaMemcpy(ho.data(), o, n * 8, cudaMemcpyDeviceToHost);
  int c0 = variant == 3 ? 0 : -2;
  int bad = 0;
  for (int m = 0; m < 5; ++m) for (int jj = 0; jj < (int)box[1]; ++jj) for (int ii = 0; ii < (int)box[0]; ++ii) {
    int i = ii + c0, j = jj + c0;
    double ex = (i >= 0 && i < nx && j >= 0 && j < ny) ? h[i + sy * j + sm_ * m] : 0.0;
    double g = ho[(m * box[1] + jj) * box[0] + ii];
    if (g != ex) { if (bad < 3) printf("mismatch m%d j%d i%d got %g exp %g\n", m, jj, ii, g, ex); bad++; }
  }
  printf("variant %d: bad=%d\n", variant, bad);
  return 0;
}

#ifndef PROBE_LIB
int main(int argc, char** argv) { return probe_main(argc > 1 ? atoi(argv[1]) : 0); }
#endif
