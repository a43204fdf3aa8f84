// Achievable HBM bandwidth of plain streaming kernels with the read/write mix
// of the repo's workloads (B200): 1 read + 1 write (copy: the MEASURED_PEAKS
// figure's shape), 2 reads + 1 write (rhs: u, forcing -> rhs), 3 reads + 1
// write (seismic dz: vz1..3 -> value_dz).  256^3 doubles per array, 16-byte
// vector loads/stores, grid = 148 x 8 CTAs of 256, best of 20 launches.
#include <cuda_runtime.h>
#include <cstdio>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s\n", cudaGetErrorString(e)); return 1; } } while (0)
template <int R>
__global__ void mix(const double2 *a, const double2 *b, const double2 *c, double2 *o, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        double2 v = __ldcs(a + i);
        if (R >= 2) { double2 w = __ldcs(b + i); v.x += w.x; v.y += w.y; }
        if (R >= 3) { double2 w = __ldcs(c + i); v.x += w.x; v.y += w.y; }
        __stcs(o + i, v);
    }
}
int main() {
    const size_t n = 256ull * 256 * 256 / 2;  // double2 elements
    double2 *a, *b, *c, *o;
    CK(cudaMalloc(&a, n * 16)); CK(cudaMalloc(&b, n * 16)); CK(cudaMalloc(&c, n * 16)); CK(cudaMalloc(&o, n * 16));
    CK(cudaMemset(a, 0, n * 16)); CK(cudaMemset(b, 0, n * 16)); CK(cudaMemset(c, 0, n * 16));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int r = 1; r <= 3; ++r) {
        float best = 1e9;
        for (int it = 0; it < 25; ++it) {
            cudaEventRecord(e0);
            if (r == 1) mix<1><<<148 * 8, 256>>>(a, b, c, o, n);
            else if (r == 2) mix<2><<<148 * 8, 256>>>(a, b, c, o, n);
            else mix<3><<<148 * 8, 256>>>(a, b, c, o, n);
            cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (it >= 5 && ms < best) best = ms;
        }
        CK(cudaGetLastError());
        const double bytes = (r + 1.0) * n * 16;
        printf("%d read(s) + 1 write: %8.2f us  %7.1f GB/s\n", r, best * 1e3, bytes / best * 1e-6);
    }
    return 0;
}
