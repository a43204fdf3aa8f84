// FP64 microbenchmarks on B200: DFMA throughput (many independent chains per
// thread, full grid) and dependent-chain latency (1 warp).  Reported in
// profiles/fp64_r01.txt; used as the FP64 co-roofline in DESIGN.md.
#include <cstdio>
#include <cuda_runtime.h>

template <int CHAINS>
__global__ void dfma_tput(double *out, int iters, double a, double b) {
    double x[CHAINS];
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) x[c] = threadIdx.x * 1e-3 + c;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int c = 0; c < CHAINS; ++c) x[c] = fma(x[c], a, b);
    }
    double s = 0;
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) s += x[c];
    if (s == 12345.678) out[0] = s;
}

__global__ void dfma_lat(double *out, long long *cyc, int iters, double a, double b) {
    double x = threadIdx.x;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        x = fma(x, a, b); x = fma(x, a, b); x = fma(x, a, b); x = fma(x, a, b);
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = t1 - t0; out[1] = x; }
}

__global__ void dadd_lat(double *out, long long *cyc, int iters, double b) {
    double x = threadIdx.x;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) { x = x + b; x = x + b; x = x + b; x = x + b; }
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = t1 - t0; out[2] = x; }
}

int main() {
    double *out; long long *cyc;
    cudaMalloc(&out, 64); cudaMalloc(&cyc, 64);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int iters = 20000, chains = 8;
    for (int threads : {256, 512, 1024}) {
        int blocks = sms * (2048 / threads);
        dfma_tput<chains><<<blocks, threads>>>(out, 100, 1.0000001, 1e-9);
        cudaEventRecord(e0);
        dfma_tput<chains><<<blocks, threads>>>(out, iters, 1.0000001, 1e-9);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        double flops = 2.0 * chains * (double)iters * blocks * threads;
        printf("DFMA throughput: %d thr/blk x %d blk: %.2f TFLOP/s  (%.1f DFMA/clk/SM at %d MHz nominal)\n",
               threads, blocks, flops / ms / 1e9, flops / 2 / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000);
    }
    long long h;
    dfma_lat<<<1, 32>>>(out, cyc, 10000, 1.0000001, 1e-9);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("DFMA dependent latency: %.2f cycles\n", h / 40000.0);
    dadd_lat<<<1, 32>>>(out, cyc, 10000, 1e-9);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("DADD dependent latency: %.2f cycles\n", h / 40000.0);
    printf("err: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
