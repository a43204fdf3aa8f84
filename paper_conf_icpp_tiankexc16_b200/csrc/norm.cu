// norm.cu -- SURVEY §8(f) f1: the NAS rhs_norm numerator, Σ rhs(m,i,j,k)^2
// over the interior points (1 <= i <= nx-2, 1 <= j <= ny-2, 1 <= k <= nz-2)
// of a field in the shared `dim` layout, per component m.  NPB error.f
// rhs_norm then takes sqrt(sum / ((nx-2)(ny-2)(nz-2))): fused into the final
// pass for a full grid (safara_rhs_rms), or a separate 1-thread-per-component
// kernel after the cross-slab NCCL all-reduce (safara_shard_rms).
//
// HBM-bound streaming reduction: each warp owns whole (m, k, j) rows, lanes
// stride i (coalesced 256 B per load), fp64 accumulation.  Deterministic: a
// fixed grid (148 x 4 blocks per component, independent of the input), fixed
// per-thread order, fixed warp/block trees, and a second one-block pass that
// sums the per-block partials in block order.
#include <cstdint>

#include "safara_internal.h"

namespace safara {
namespace {

constexpr int NORM_THREADS = 256;
constexpr int NORM_WARPS = NORM_THREADS / 32;

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    return v;
}

// blockIdx.y = component m; block b of gridDim.x takes rows
// [b*R/G, (b+1)*R/G) of the R = nk*(ny-2) interior rows of that component.
__global__ void __launch_bounds__(NORM_THREADS)
sumsq_partial(const double *__restrict__ rhs, int nx, int ny, int sy, int sm, int sk, int kl0,
              int nk, double *__restrict__ work) {
    const int m = blockIdx.y, G = gridDim.x, b = blockIdx.x;
    const long long R = (long long)nk * (ny - 2);
    const long long r0 = R * b / G, r1 = R * (b + 1) / G;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    double acc = 0.0;
    for (long long r = r0 + warp; r < r1; r += NORM_WARPS) {
        const int kk = (int)(r / (ny - 2)), j = 1 + (int)(r % (ny - 2));
        const double *row = rhs + ((long long)sy * j + (long long)sm * m + (long long)sk * (kl0 + kk));
        for (int i = 1 + lane; i <= nx - 2; i += 32) {
            const double v = __ldcs(row + i);
            acc = fma(v, v, acc);
        }
    }
    acc = warp_sum(acc);
    __shared__ double s[NORM_WARPS];
    if (lane == 0) s[warp] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < NORM_WARPS; ++w) t += s[w];
        work[m * G + b] = t;
    }
}

// one block: warp m sums component m's G partials in a fixed order; with
// npts > 0 it also finishes NPB rhs_norm: out[m] = sqrt(sum / npts)
__global__ void sumsq_final(const double *__restrict__ work, int G, double *__restrict__ out,
                            double npts) {
    const int m = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (m >= 5) return;
    double t = 0.0;
    for (int b = lane; b < G; b += 32) t += work[m * G + b];
    t = warp_sum(t);
    if (lane == 0) out[m] = npts > 0.0 ? sqrt(t / npts) : t;
}

// NPB error.f rhs_norm's last step on summed numerators (after the
// cross-slab all-reduce): v[m] = sqrt(v[m] / npts)
__global__ void rms_finish(double *__restrict__ v, double npts) {
    const int m = threadIdx.x;
    if (m < 5) v[m] = sqrt(v[m] / npts);
}

}  // namespace

int norm_grid() { return 148 * 4; }

cudaError_t launch_sumsq(const double *rhs, int nx, int ny, int sy, int sm, int sk, int kl0, int nk,
                         double *work, double *out, cudaStream_t s, double npts) {
    const int G = norm_grid();
    sumsq_partial<<<dim3(G, 5), NORM_THREADS, 0, s>>>(rhs, nx, ny, sy, sm, sk, kl0, nk, work);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    sumsq_final<<<1, 5 * 32, 0, s>>>(work, G, out, npts);
    return cudaGetLastError();
}

cudaError_t launch_partials_final(const double *work, int G, double *out, double npts,
                                  cudaStream_t s) {
    sumsq_final<<<1, 5 * 32, 0, s>>>(work, G, out, npts);
    return cudaGetLastError();
}

cudaError_t launch_rms_finish(double *v, double npts, cudaStream_t s) {
    rms_finish<<<1, 32, 0, s>>>(v, npts);
    return cudaGetLastError();
}

}  // namespace safara
