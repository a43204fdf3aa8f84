// Memory-space access latencies on this B200, for SAFARA's L x C cost model
// (§III-B3: "we measured the latencies with the
// microbenchmarks of [19]").  Dependent pointer chasing by
// one thread, clock64() around the chain, so each load waits for the
// previous one:
//   register  dependent DFMA / DADD chains (ALU latency, the "register" row)
//   shared    ld.shared chain through a permutation in shared memory
//   l1        ld.global chain over an 8 KB working set (L1 hits after warm-up)
//   l2        ld.global.cg chain over 16 MB (L2 hits: bypasses L1, fits 126 MB L2)
//   dram      ld.global.cg chain over 1 GB with a 4 KB+ stride permutation (misses)
//   uncoalesced: one warp, each lane chasing its own chain 4 KB apart
//                (32 sectors per warp load; the average per-load latency)
// Output: one JSON object (cycles per load, SM clock domain).
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <vector>

__global__ void alu_lat(double *out, long long *cyc, int iters) {
    double x = threadIdx.x + 1.0, y = 1.0000001;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) { x = fma(x, y, 1e-9); x = fma(x, y, 1e-9); }
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = t1 - t0; out[0] = x; }
}

__global__ void smem_lat(long long *cyc, unsigned *sink, int iters) {
    __shared__ unsigned nxt[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) nxt[i] = (i * 1021u + 7u) % 4096u;
    __syncthreads();
    if (threadIdx.x) return;
    unsigned p = 0;
    for (int i = 0; i < 64; ++i) p = nxt[p];
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) p = nxt[p];
    long long t1 = clock64();
    cyc[0] = t1 - t0;
    sink[0] = p;
}

template <bool CG>
__global__ void chase(const unsigned long long *nxt, long long *cyc, unsigned long long *sink,
                      int warm, int iters) {
    unsigned long long p = 0;
    for (int i = 0; i < warm; ++i) p = CG ? __ldcg(nxt + p) : nxt[p];
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) p = CG ? __ldcg(nxt + p) : nxt[p];
    long long t1 = clock64();
    cyc[0] = t1 - t0;
    sink[0] = p;
}

// 32 lanes, each its own chain; lane chains are `lane_stride` elements apart
__global__ void chase_warp(const unsigned long long *nxt, long long *cyc,
                           unsigned long long *sink, int iters, long long lane_stride) {
    unsigned long long p = (unsigned long long)(threadIdx.x * lane_stride);
    for (int i = 0; i < 16; ++i) p = __ldcg(nxt + p);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) p = __ldcg(nxt + p);
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
    sink[threadIdx.x] = p;
}

// a single cycle through n elements, consecutive hops `stride` elements apart
static std::vector<unsigned long long> ring(size_t n, size_t stride) {
    std::vector<unsigned long long> v(n);
    const size_t hops = n / stride;
    for (size_t h = 0; h < hops; ++h) {
        const size_t a = h * stride, b = ((h + 1) % hops) * stride;
        for (size_t o = 0; o < stride; ++o) v[a + o] = b + o;  // any offset stays on the ring
    }
    return v;
}

static double run_chase(size_t bytes, size_t stride_bytes, bool cg, int iters) {
    const size_t n = bytes / 8, stride = stride_bytes / 8;
    std::vector<unsigned long long> h = ring(n, stride);
    unsigned long long *d, *sink;
    long long *cyc, hc = 0;
    cudaMalloc(&d, n * 8);
    cudaMalloc(&sink, 256 * 8);
    cudaMalloc(&cyc, 8);
    cudaMemcpy(d, h.data(), n * 8, cudaMemcpyHostToDevice);
    const int warm = (int)((n / stride) < 100000 ? n / stride : 0);
    if (cg) chase<true><<<1, 1>>>(d, cyc, sink, warm, iters);
    else chase<false><<<1, 1>>>(d, cyc, sink, warm, iters);
    cudaMemcpy(&hc, cyc, 8, cudaMemcpyDeviceToHost);
    cudaFree(d); cudaFree(sink); cudaFree(cyc);
    return (double)hc / iters;
}

int main() {
    double *out;
    long long *cyc, hc;
    unsigned *usink;
    cudaMalloc(&out, 64);
    cudaMalloc(&cyc, 64);
    cudaMalloc(&usink, 64);
    alu_lat<<<1, 32>>>(out, cyc, 20000);
    cudaMemcpy(&hc, cyc, 8, cudaMemcpyDeviceToHost);
    const double reg = hc / 40000.0;
    smem_lat<<<1, 256>>>(cyc, usink, 20000);
    cudaMemcpy(&hc, cyc, 8, cudaMemcpyDeviceToHost);
    const double sh = hc / 20000.0;
    const double l1 = run_chase(8 << 10, 128, false, 20000);
    const double l2 = run_chase(16 << 20, 256, true, 20000);
    const double dram = run_chase(1ull << 30, 4096 + 64, true, 4000);
    // uncoalesced: 32 lanes, chains 64 KB apart inside a 1 GB ring
    double unc = 0;
    {
        const size_t n = (1ull << 30) / 8, stride = (4096 + 64) / 8;
        std::vector<unsigned long long> h = ring(n, stride);
        unsigned long long *d, *sink;
        cudaMalloc(&d, n * 8);
        cudaMalloc(&sink, 256 * 8);
        cudaMemcpy(d, h.data(), n * 8, cudaMemcpyHostToDevice);
        chase_warp<<<1, 32>>>(d, cyc, sink, 2000, (long long)stride * 997);
        cudaMemcpy(&hc, cyc, 8, cudaMemcpyDeviceToHost);
        unc = hc / 2000.0;
        cudaFree(d); cudaFree(sink);
    }
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("{\"register\": %.1f, \"shared\": %.1f, \"l1\": %.1f, \"l2\": %.1f, \"dram\": %.1f, "
           "\"global_uncoalesced\": %.1f, \"unit\": \"SM cycles per dependent access\", "
           "\"sm_clock_mhz_nominal\": %d, \"err\": \"%s\"}\n",
           reg, sh, l1, l2, dram, unc, clk / 1000, cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
