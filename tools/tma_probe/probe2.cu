// TMA probe with runtime-configurable block size / smem size / offsets.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
__device__ __forceinline__ uint32_t s32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void __launch_bounds__(320, 1) probe(const __grid_constant__ CUtensorMap tmap, double* out, int n, int buf_off, int bar_off) {
  extern __shared__ __align__(128) unsigned char sm[];
  double* buf = (double*)(sm + buf_off);
  uint64_t* bar = (uint64_t*)(sm + bar_off);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(s32(bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(s32(bar)), "r"(n * 8) : "memory");
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
      :: "r"(s32(buf)), "l"((uint64_t)&tmap), "r"(-1), "r"(-1), "r"(0), "r"(1), "r"(s32(bar)) : "memory");
  }
  uint32_t done = 0;
  do {
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(s32(bar)), "r"(0) : "memory");
  } while (!done);
  for (int t = threadIdx.x; t < n; t += blockDim.x) out[t] = buf[t];
}
int main(int argc, char** argv) {
  int nthr = atoi(argv[1]); int smem = atoi(argv[2]); int buf_off = atoi(argv[3]); int bar_off = atoi(argv[4]);
  int nblk = argc > 5 ? atoi(argv[5]) : 1;
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
  cuuint64_t gdim[4] = {(cuuint64_t)nx, (cuuint64_t)ny, 5, (cuuint64_t)nz};
  cuuint64_t gstr[3] = {(cuuint64_t)sy * 8, sm_ * 8, sk * 8};
  cuuint32_t box[4] = {36, 14, 5, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, d, gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  int n = 36 * 14 * 5;
  cudaError_t e0 = cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  probe<<<nblk, nthr, smem>>>(map, o, n, buf_off, bar_off);
  cudaError_t e1 = cudaGetLastError();
  cudaError_t e = cudaDeviceSynchronize();
  printf("thr=%d smem=%d buf=%d bar=%d blk=%d: enc=%d attr=%s launch=%s sync=%s\n", nthr, smem, buf_off, bar_off, nblk, (int)r,
         cudaGetErrorString(e0), cudaGetErrorString(e1), cudaGetErrorString(e));
  return 0;
}
