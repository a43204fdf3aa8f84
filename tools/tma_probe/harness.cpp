// Calls libsafara_rhs.so directly (no Python/torch): one 12^3 pass.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "safara.h"
int main(int argc, char** argv) {
  int n = argc > 1 ? atoi(argv[1]) : 12;
  int flags = argc > 2 ? atoi(argv[2]) : 1;
  printf("init=%d\n", safara_rhs_init(0));
  safara_dims_t d; safara_dims_canonical(n, n, n, &d);
  size_t cnt = (size_t)d.sk * n;
  std::vector<double> h(cnt);
  for (size_t t = 0; t < cnt; ++t) h[t] = 1.0 + 0.001 * (t % 97);
  double *u, *f, *r;
  cudaMalloc(&u, cnt * 8); cudaMalloc(&f, cnt * 8); cudaMalloc(&r, cnt * 8);
  cudaMemcpy(u, h.data(), cnt * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(f, h.data(), cnt * 8, cudaMemcpyHostToDevice);
  safara_coeffs_t c; safara_coeffs_nas(n, n, n, 0.01, &c);
  int rc = safara_rhs_ex(u, f, r, &d, &c, flags, nullptr);
  cudaError_t e = cudaDeviceSynchronize();
  printf("rc=%d sync=%s\n", rc, cudaGetErrorString(e));
  return 0;
}
