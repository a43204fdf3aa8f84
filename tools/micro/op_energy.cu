// Dynamic energy per warp instruction on the B200 (NVML total-energy counter
// minus the idle power over the same time): DFMA, DMUL-free integer ops,
// LDS.64 and LDS.128, FFMA -- the unit costs behind the rhs kernel's energy
// budget (the bench is power-capped at 1 kW).
// usage: op_energy [seconds] [idle_watts]
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <cstdio>
#include <cstdlib>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
constexpr int IT = 4096;

__global__ void k_dfma(double *out, double a, double b) {
    double x[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = threadIdx.x * 1e-3 + c;
    for (int i = 0; i < IT; ++i) {
#pragma unroll
        for (int c = 0; c < 8; ++c) x[c] = fma(x[c], a, b);
    }
    double s = 0;
#pragma unroll
    for (int c = 0; c < 8; ++c) s += x[c];
    if (s == 1.2345) out[0] = s;
}
__global__ void k_ffma(float *out, float a, float b) {
    float x[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = threadIdx.x * 1e-3f + c;
    for (int i = 0; i < IT; ++i) {
#pragma unroll
        for (int c = 0; c < 8; ++c) x[c] = fmaf(x[c], a, b);
    }
    float s = 0;
#pragma unroll
    for (int c = 0; c < 8; ++c) s += x[c];
    if (s == 1.2345f) out[0] = s;
}
__global__ void k_int(unsigned *out, unsigned a, unsigned b) {
    unsigned x[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = threadIdx.x + c;
    for (int i = 0; i < IT; ++i) {
#pragma unroll
        for (int c = 0; c < 8; ++c) x[c] = x[c] * a + b;
    }
    unsigned s = 0;
#pragma unroll
    for (int c = 0; c < 8; ++c) s ^= x[c];
    if (s == 12345u) out[0] = s;
}
template <int W>  // W = 1: LDS.64, 2: LDS.128
__global__ void k_lds(double *out) {
    __shared__ double sm[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = i;
    __syncthreads();
    unsigned long long acc = 0;
    int base = threadIdx.x * W;
    for (int i = 0; i < IT; ++i) {
        const int o = (base + (i & 7) * 256 * W) & (4096 - 1);
        if (W == 1) {
            double v;
            asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"((unsigned)__cvta_generic_to_shared(sm + o)));
            acc ^= __double_as_longlong(v);
        } else {
            double v0, v1;
            asm volatile("ld.shared.v2.f64 {%0,%1}, [%2];" : "=d"(v0), "=d"(v1) : "r"((unsigned)__cvta_generic_to_shared(sm + o)));
            acc ^= __double_as_longlong(v0) ^ __double_as_longlong(v1);
        }
    }
    if (acc == 12345ull) out[0] = (double)acc;
}

typedef int (*nvmlInit_t)();
typedef int (*nvmlGetHandle_t)(unsigned, void **);
typedef int (*nvmlEnergy_t)(void *, unsigned long long *);
typedef int (*nvmlClock_t)(void *, int, unsigned *);

int main(int argc, char **argv) {
    const double secs = argc > 1 ? atof(argv[1]) : 2.0;
    const double idle_w = argc > 2 ? atof(argv[2]) : 248.0;
    void *h = dlopen("libnvidia-ml.so.1", RTLD_NOW);
    if (!h) { printf("no NVML\n"); return 1; }
    void *dev;
    ((nvmlInit_t)dlsym(h, "nvmlInit_v2"))();
    ((nvmlGetHandle_t)dlsym(h, "nvmlDeviceGetHandleByIndex_v2"))(0, &dev);
    auto energy = (nvmlEnergy_t)dlsym(h, "nvmlDeviceGetTotalEnergyConsumption");
    auto clock = (nvmlClock_t)dlsym(h, "nvmlDeviceGetClockInfo");
    double *d; CK(cudaMalloc(&d, 64));
    const int grid = 148 * 4, block = 256;
    // warp instructions of the measured op per launch (the loop body; the
    // loop's own IADD/ISETP/BRA are 3 per 8 ops and counted separately)
    const double warps = grid * block / 32.0;
    const char *names[] = {"DFMA", "FFMA", "IMAD", "LDS.64 (+xor)", "LDS.128 (+2 xor)"};
    for (int rep = 0; rep < 2; ++rep)
        for (int t = 0; t < 5; ++t) {
            auto launch = [&]() {
                if (t == 0) k_dfma<<<grid, block>>>(d, 1.0000001, 1e-9);
                else if (t == 1) k_ffma<<<grid, block>>>((float *)d, 1.0001f, 1e-6f);
                else if (t == 2) k_int<<<grid, block>>>((unsigned *)d, 3u, 7u);
                else if (t == 3) k_lds<1><<<grid, block>>>(d);
                else k_lds<2><<<grid, block>>>(d);
            };
            const double ops = warps * IT * (t <= 2 ? 8.0 : 1.0);
            cudaEvent_t e0, e1;
            CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
            for (int w = 0; w < 5; ++w) launch();
            CK(cudaEventRecord(e0));
            for (int w = 0; w < 10; ++w) launch();
            CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
            float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
            const int K = (int)(secs * 1e3 / (ms / 10)) + 1;
            for (int w = 0; w < K / 2; ++w) launch();
            CK(cudaDeviceSynchronize());
            unsigned long long j0, j1;
            energy(dev, &j0);
            CK(cudaEventRecord(e0));
            for (int w = 0; w < K; ++w) launch();
            CK(cudaEventRecord(e1));
            unsigned clk = 0; clock(dev, 1, &clk);
            CK(cudaEventSynchronize(e1));
            energy(dev, &j1);
            CK(cudaEventElapsedTime(&ms, e0, e1));
            const double us = ms * 1e3 / K, mj = (double)(j1 - j0) / K, w = mj / us * 1e3;
            const double dyn_pj = (mj - idle_w * us * 1e-3) * 1e9 / ops;
            printf("%-18s %9.1f us  %6.1f W  %5u MHz  %7.3f Twarp-inst/s  dynamic %7.1f pJ/warp-inst (%5.2f pJ/lane-op)\n",
                   names[t], us, w, clk, ops / us * 1e-6, dyn_pj, dyn_pj / 32);
            fflush(stdout);
        }
    return 0;
}
