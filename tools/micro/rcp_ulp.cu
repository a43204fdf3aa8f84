// rcp_ulp.cu -- accuracy of the production reciprocal variants (rhs_kernel.cuh
// recip(), SAFARA_RCP 0/1/2) against the correctly rounded IEEE 1.0/x, over
// the density range of the NAS fields (u1 in [0.5, 32], a superset of the
// [2, 15.8] seen at class C) plus random exponents.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o rcp_ulp rcp_ulp.cu
#include <cstdio>
#include <cstdint>
#include <cstring>

__device__ double rcp_seed(double x) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    return r;
}
__device__ double v0(double x) {  // 3 Newton steps
    double r = rcp_seed(x), e;
    e = __fma_rn(-x, r, 1.0); r = __fma_rn(r, e, r);
    e = __fma_rn(-x, r, 1.0); r = __fma_rn(r, e, r);
    e = __fma_rn(-x, r, 1.0); return __fma_rn(r, e, r);
}
__device__ double v1(double x) {  // 2 Newton steps
    double r = rcp_seed(x), e;
    e = __fma_rn(-x, r, 1.0); r = __fma_rn(r, e, r);
    e = __fma_rn(-x, r, 1.0); return __fma_rn(r, e, r);
}
__device__ double v2(double x) {  // one cubic step
    const double r = rcp_seed(x);
    const double e = __fma_rn(-x, r, 1.0);
    return __fma_rn(r, __fma_rn(e, e, e), r);
}

__device__ unsigned long long mix(unsigned long long z) {
    z += 0x9e3779b97f4a7c15ull;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}

__global__ void k(long long n, unsigned long long *maxulp, unsigned long long *cnt, int wide) {
    unsigned long long m[4] = {0, 0, 0, 0}, c[4] = {0, 0, 0, 0};
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < n;
         t += (long long)gridDim.x * blockDim.x) {
        const unsigned long long h = mix((unsigned long long)t);
        double x;
        if (wide) {  // random mantissa, exponent in [-60, 60]
            const unsigned long long bits = (h & 0x000fffffffffffffull) |
                                            ((unsigned long long)(1023 - 60 + (int)((h >> 52) % 121)) << 52);
            memcpy(&x, &bits, 8);
        } else {
            x = 0.5 + 31.5 * ((h >> 11) * 0x1.0p-53);
        }
        const double ref = 1.0 / x;
        const double got[3] = {v0(x), v1(x), v2(x)};
        long long rb;
        memcpy(&rb, &ref, 8);
        for (int v = 0; v < 3; ++v) {
            long long gb;
            memcpy(&gb, &got[v], 8);
            const unsigned long long d = (unsigned long long)(gb > rb ? gb - rb : rb - gb);
            if (d > m[v]) m[v] = d;
            if (d) c[v]++;
        }
    }
    for (int v = 0; v < 3; ++v) {
        atomicMax(&maxulp[v], m[v]);
        atomicAdd(&cnt[v], c[v]);
    }
}

int main() {
    unsigned long long *d;
    cudaMalloc(&d, 6 * sizeof(unsigned long long));
    const long long n = 1LL << 30;
    for (int wide = 0; wide < 2; ++wide) {
        cudaMemset(d, 0, 6 * sizeof(unsigned long long));
        k<<<148 * 8, 256>>>(n, d, d + 3, wide);
        unsigned long long h[6];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        const char *nm[3] = {"3 Newton (6 DFMA)", "2 Newton (4 DFMA)", "cubic (3 DFMA)"};
        printf("%s inputs, n = %lld\n", wide ? "wide-exponent" : "u1 in [0.5, 32]", n);
        for (int v = 0; v < 3; ++v)
            printf("  %-20s max |ulp| vs 1.0/x = %llu, inexact-vs-IEEE count = %llu (%.3g)\n", nm[v],
                   h[v], h[3 + v], (double)h[3 + v] / n);
    }
    return 0;
}
