// DRAM-sourced TMA streaming like the rhs kernel: CTA c streams column tile
// (c % 70) over its half of 162 planes, boxes u(38x16x5) + f(34x12x5) per
// plane, S-stage ring; `pad_kb` extra dynamic smem emulates the L1 squeeze.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>

__device__ __forceinline__ uint32_t s32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void stream(const __grid_constant__ CUtensorMap um, const __grid_constant__ CUtensorMap fm,
                       int S, int slot, int planes, int mode) {
  extern __shared__ __align__(1024) unsigned char sm[];
  uint64_t* bar = (uint64_t*)(sm + (size_t)S * slot);
  const int tile = blockIdx.x % 70, part = blockIdx.x / 70;
  const int i0 = 1 + (tile % 5) * 32, j0 = 1 + (tile / 5) * 12, k0 = 1 + part * planes;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(s32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int it) {
    int s = it % S;
    unsigned char* dst = sm + (size_t)s * slot;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(s32(&bar[s])), "r"(24320 + 16320) : "memory");
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
      :: "r"(s32(dst)), "l"((uint64_t)&um), "r"(i0 - 3), "r"(j0 - 2), "r"(0), "r"(k0 + it), "r"(s32(&bar[s])) : "memory");
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
      :: "r"(s32(dst + 24320)), "l"((uint64_t)&fm), "r"(i0 - 1), "r"(j0), "r"(0), "r"(k0 + it), "r"(s32(&bar[s])) : "memory");
  };
  if (threadIdx.x == 0) for (int it = 0; it < S && it < planes; ++it) issue(it);
  double acc = 0;
  if (mode == 1) {
    // the rhs kernel's protocol: each warp waits for plane it+2 (lead 2), reads,
    // then releases plane it with an atomic; the last warp refills with it+S
    __shared__ unsigned cnt[8];
    if (threadIdx.x < 8) cnt[threadIdx.x] = 0;
    __syncthreads();
    const int nw = blockDim.x / 32, lane = threadIdx.x % 32;
    for (int it = 0; it < planes; ++it) {
      int w = it + 2 < planes ? it + 2 : planes - 1;
      { int s = w % S; uint32_t par = (w / S) & 1; uint32_t done = 0;
        do { asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(s32(&bar[s])), "r"(par) : "memory"); } while (!done); }
      acc += ((const double*)(sm + (size_t)(it % S) * slot))[threadIdx.x];
      __syncwarp();
      if (lane == 0) {
        __threadfence_block();
        unsigned old = atomicAdd(&cnt[it % S], 1u);
        if (old == (unsigned)(nw - 1)) { cnt[it % S] = 0; __threadfence_block(); if (it + S < planes) issue(it + S); }
      }
    }
    if (acc == 1.2345) printf("x");
    return;
  }
  for (int it = 0; it < planes; ++it) {
    int s = it % S; uint32_t par = (it / S) & 1; uint32_t done = 0;
    do { asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(s32(&bar[s])), "r"(par) : "memory"); } while (!done);
    acc += ((const double*)(sm + (size_t)s * slot))[threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0 && it + S < planes) issue(it + S);
  }
  if (acc == 1.2345) printf("x");
}

int main() {
  const int NX = 168, NY = 162, K = 162;
  size_t elems = (size_t)NX * NY * 5 * K;
  double *u, *f, *flush;
  cudaMalloc(&u, elems * 8); cudaMalloc(&f, elems * 8); cudaMalloc(&flush, 512ull << 20);
  cudaMemset(u, 0, elems * 8); cudaMemset(f, 0, elems * 8);
  void* fn = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  CUtensorMap um, fm;
  cuuint64_t gdim[4] = {162, (cuuint64_t)NY, 5, (cuuint64_t)K};
  cuuint64_t gstr[3] = {(cuuint64_t)NX * 8, (cuuint64_t)NX * NY * 8, (cuuint64_t)NX * NY * 5 * 8};
  cuuint32_t bu[4] = {38, 16, 5, 1}, bf[4] = {34, 12, 5, 1}, es[4] = {1, 1, 1, 1};
  enc(&um, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, u, gdim, gstr, bu, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  enc(&fm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, f, gdim, gstr, bf, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int slot = 40960;
  for (int mode : {0, 1}) for (int S : {3, 4, 5}) for (int pad_kb : {0, 48}) {
    int smem = S * slot + 1024 + pad_kb * 1024;
    if (smem > 227 * 1024) continue;
    cudaFuncSetAttribute(stream, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    float best = 1e9;
    for (int rep = 0; rep < 3; ++rep) {
      cudaMemset(flush, rep, 512ull << 20);
      cudaEventRecord(e0);
      stream<<<140, 384, smem>>>(um, fm, S, slot, 80, mode);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    double bytes = 140.0 * 80 * 40640;
    printf("mode=%d S=%d smem=%3d KB (L1 left ~%3d KB): %6.1f us  %6.0f GB/s (L2->SM incl halo)  err=%s\n", mode, S, smem / 1024,
           228 - smem / 1024, best * 1e3, bytes / best / 1e6, cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
