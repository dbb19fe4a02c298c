// fp64_micro.cu -- B200 fp64 pipe micro-benchmarks:
// DFMA / DADD / DMUL / DMNMX throughput and the cost of IEEE fp64 divide,
// sqrt and rsqrt() in DFMA-slot equivalents.  Build and run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_micro tools/fp64_micro.cu && ./fp64_micro
#include <cstdio>
#include <cuda_runtime.h>

#define ILP 8
#define ITERS 4096

template <int OP>
__global__ void k(double* out, double a, double b) {
  double x[ILP];
#pragma unroll
  for (int i = 0; i < ILP; ++i) x[i] = a + threadIdx.x * 1e-9 + i * 1e-7;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < ILP; ++i) {
      if (OP == 0) x[i] = fma(x[i], a, b);
      if (OP == 1) x[i] = x[i] + b;
      if (OP == 2) x[i] = x[i] * a;
      if (OP == 3) x[i] = fmax(x[i], b) - a;  // DMNMX + DADD
      if (OP == 4) x[i] = b / x[i];
      if (OP == 5) x[i] = sqrt(x[i]) + b;
      if (OP == 6) x[i] = rsqrt(x[i]) + b;
    }
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < ILP; ++i) s += x[i];
  if (s == 12345.678) out[0] = s;
}

// dependent-chain latency (one warp per SM, ILP 1), cycles per op by clock64
template <int OP>
__global__ void k_lat(double* out, long long* cyc, double a, double b) {
  double x = a + threadIdx.x * 1e-12;
  const long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
    if (OP == 0) x = fma(x, a, b);
    if (OP == 1) x = x + b;
    if (OP == 2) x = x * a;
    if (OP == 3) {
      double y;
      asm volatile("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
      x = y + b;
    }
  }
  const long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  if (x == 12345.678) out[0] = x;
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  int sms = p.multiProcessorCount;
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"clock_khz_attr\": %d, \"results\": [\n", p.name, sms, clk);
  double* out;
  cudaMalloc(&out, 8);
  const char* names[] = {"dfma", "dadd", "dmul", "dmnmx+dadd", "ddiv", "dsqrt+dadd", "rsqrt+dadd"};
  const int threads = 256;
  for (int op = 0; op < 7; ++op) {
    for (int bps = 4; bps <= 8; bps *= 2) {
      int blocks = sms * bps;
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      auto launch = [&]() {
        switch (op) {
          case 0: k<0><<<blocks, threads>>>(out, 1.0000001, 1e-9); break;
          case 1: k<1><<<blocks, threads>>>(out, 1.0000001, 1e-9); break;
          case 2: k<2><<<blocks, threads>>>(out, 1.0000001, 1e-9); break;
          case 3: k<3><<<blocks, threads>>>(out, 1e-12, 0.5); break;
          case 4: k<4><<<blocks, threads>>>(out, 1.0, 1.0); break;
          case 5: k<5><<<blocks, threads>>>(out, 1.0, 1e-3); break;
          case 6: k<6><<<blocks, threads>>>(out, 1.0, 1e-3); break;
        }
      };
      launch();
      cudaDeviceSynchronize();
      float best = 1e30f;
      for (int r = 0; r < 5; ++r) {
        cudaEventRecord(e0);
        launch();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      double ops = (double)blocks * threads * ITERS * ILP;
      double gops = ops / (best * 1e-3) / 1e9;
      printf("  {\"op\": \"%s\", \"blocks_per_sm\": %d, \"ms\": %.4f, \"Gop_per_s\": %.1f, \"op_per_clk_per_sm_at_1965\": %.2f}%s\n",
             names[op], bps, best, gops, gops * 1e9 / (sms * 1.965e9), (op == 6 && bps == 8) ? "" : ",");
    }
  }
  printf("], \"latency_cycles\": [\n");
  {
    long long* cyc;
    cudaMalloc(&cyc, sizeof(long long) * sms);
    const char* ln[] = {"dfma", "dadd", "dmul", "mufu.rsq64h+dadd"};
    for (int op = 0; op < 4; ++op) {
      for (int r = 0; r < 2; ++r) {
        switch (op) {
          case 0: k_lat<0><<<sms, 32>>>(out, cyc, 1.0000001, 1e-9); break;
          case 1: k_lat<1><<<sms, 32>>>(out, cyc, 1.0000001, 1e-9); break;
          case 2: k_lat<2><<<sms, 32>>>(out, cyc, 1.0000001, 1e-9); break;
          case 3: k_lat<3><<<sms, 32>>>(out, cyc, 1.0, 1.0); break;
        }
        cudaDeviceSynchronize();
      }
      long long c = 0;
      cudaMemcpy(&c, cyc, sizeof c, cudaMemcpyDeviceToHost);
      printf("  {\"op\": \"%s\", \"cycles_per_dependent_op\": %.2f}%s\n", ln[op], (double)c / ITERS,
             op == 3 ? "" : ",");
    }
  }
  printf("]}\n");
  return 0;
}
