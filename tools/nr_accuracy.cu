// Accuracy of the Newton-refined hardware rsqrt / rcp used by the sweeps
// (pf_model.cuh rsqrt_nr / rcp_nr, copied here verbatim as test code):
// max error in ulps against the correctly rounded 1/sqrt(x) and 1/x over
// log-uniform random x in [1e-300, 1e300] and uniform x in [0.5, 2].
#include <cstdio>
#include <cmath>
#include <cstdint>

__device__ __forceinline__ double rsqrt_nr(double x) {
  double y;
  asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  const double e = fma(-x * y, y, 1.0);
  return fma(y * e, fma(0.375, e, 0.5), y);
}
__device__ __forceinline__ double rcp_nr(double x) {
  double y;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  const double e = fma(-x, y, 1.0);
  return fma(y, fma(e, e, e), y);
}
__device__ __forceinline__ double approx_rsqrt(double x) {
  double y; asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x)); return y;
}
__device__ __forceinline__ double approx_rcp(double x) {
  double y; asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x)); return y;
}
__device__ uint64_t mix(uint64_t z) {
  z += 0x9e3779b97f4a7c15ull; z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull; return z ^ (z >> 31);
}
__device__ long long ulps(double a, double b) {
  long long ia = __double_as_longlong(a), ib = __double_as_longlong(b);
  return ia > ib ? ia - ib : ib - ia;
}
__global__ void k(int mode, long long n, unsigned long long* out, double* rel) {
  long long u0 = 0, u1 = 0; double r0 = 0, r1 = 0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    double t = (mix(i * 2 + mode) >> 11) * 0x1p-53;
    double x = mode == 0 ? pow(10.0, -300.0 + 600.0 * t) : 0.5 + 1.5 * t;
    double rs = 1.0 / sqrt(x), rc = 1.0 / x;
    long long a = ulps(rsqrt_nr(x), rs), b = ulps(rcp_nr(x), rc);
    u0 = a > u0 ? a : u0; u1 = b > u1 ? b : u1;
    double e0 = fabs(approx_rsqrt(x) / rs - 1.0), e1 = fabs(approx_rcp(x) / rc - 1.0);
    r0 = e0 > r0 ? e0 : r0; r1 = e1 > r1 ? e1 : r1;
  }
  atomicMax(&out[0], (unsigned long long)u0); atomicMax(&out[1], (unsigned long long)u1);
  atomicMax((unsigned long long*)&rel[0], (unsigned long long)__double_as_longlong(r0));
  atomicMax((unsigned long long*)&rel[1], (unsigned long long)__double_as_longlong(r1));
}
int main() {
  unsigned long long* d; double* r; cudaMalloc(&d, 16); cudaMalloc(&r, 16);
  printf("{");
  for (int mode = 0; mode < 2; ++mode) {
    cudaMemset(d, 0, 16); cudaMemset(r, 0, 16);
    long long n = 1ll << 30;
    k<<<148 * 8, 256>>>(mode, n, d, r);
    unsigned long long h[2]; double hr[2];
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost); cudaMemcpy(hr, r, 16, cudaMemcpyDeviceToHost);
    printf("%s\"%s\": {\"samples\": %lld, \"rsqrt_nr_max_ulp\": %llu, \"rcp_nr_max_ulp\": %llu, "
           "\"rsqrt_approx_max_rel\": %.3e, \"rcp_approx_max_rel\": %.3e}", mode ? ", " : "",
           mode ? "uniform_0.5_2" : "logu_1e-300_1e300", n, h[0], h[1], hr[0], hr[1]);
  }
  printf("}\n");
  return cudaDeviceSynchronize() != cudaSuccess;
}
