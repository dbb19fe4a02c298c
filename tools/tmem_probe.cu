// tmem_probe.cu -- tensor memory (TMEM) as per-thread scratch from plain SIMT
// code on sm_100a: tcgen05.alloc / st / ld / dealloc without any MMA.  Checks
// that a value stored by a thread comes back bitwise, and measures the
// store + load round trip of 64 doubles per thread (the size of the mu-sweep's
// carried state) at 2 and 3 CTAs of 4 warps per SM.  Prints one JSON line.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tmem_probe tools/tmem_probe.cu
#include <cuda_runtime.h>

#include <cstdio>

__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

// 32 lanes x 32 columns of 32 bit: one tcgen05.st / ld of 32 registers per thread
__device__ __forceinline__ void tm_st32(unsigned taddr, const unsigned (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31, %32};\n" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
      "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
      "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}
__device__ __forceinline__ void tm_ld32(unsigned taddr, unsigned (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];\n"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr)
      : "memory");
}
__device__ __forceinline__ void tm_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory"); }
__device__ __forceinline__ void tm_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory"); }

template <int NCOL>
__global__ void __launch_bounds__(128) k_tmem(double* out, int iters, unsigned long long* bad) {
  __shared__ unsigned tbase;
  const int w = threadIdx.x >> 5;
  if (w == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(&tbase)),
                 "n"(NCOL));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
  const unsigned t0 = tbase + ((unsigned)(32 * (w & 3)) << 16);  // this warp's lane quarter
  double acc = 0.0;
  unsigned long long nbad = 0;
  for (int it = 0; it < iters; ++it) {
    // 64 doubles = 128 columns per thread, in 4 stores of 32 columns
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      unsigned r[32];
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        const double v = (double)(it * 1000 + q * 100 + j) + threadIdx.x * 1e-3 + blockIdx.x * 1e-7;
        const unsigned long long b = (unsigned long long)__double_as_longlong(v);
        r[2 * j] = (unsigned)b;
        r[2 * j + 1] = (unsigned)(b >> 32);
      }
      tm_st32(t0 + 32 * q, r);
    }
    tm_wait_st();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      unsigned r[32];
      tm_ld32(t0 + 32 * q, r);
      tm_wait_ld();
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        const double v = __longlong_as_double((long long)(((unsigned long long)r[2 * j + 1] << 32) | r[2 * j]));
        const double e = (double)(it * 1000 + q * 100 + j) + threadIdx.x * 1e-3 + blockIdx.x * 1e-7;
        nbad += v != e;
        acc += v;
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
  __syncthreads();
  if (w == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tbase), "n"(NCOL));
  if (nbad) atomicAdd(bad, nbad);
  if (acc == 1.2345) out[0] = acc;
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  const int sms = p.multiProcessorCount;
  double* out;
  unsigned long long* bad;
  cudaMalloc(&out, 8);
  cudaMalloc(&bad, 8);
  printf("{\"probe\": \"TMEM scratch from SIMT code\", \"results\": [");
  bool first = true;
  for (int ctas : {2, 3}) {
    cudaMemset(bad, 0, 8);
    const int iters = 2000;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_tmem<128><<<sms * ctas, 128>>>(out, 10, bad);
    cudaError_t err = cudaDeviceSynchronize();
    cudaEventRecord(e0);
    k_tmem<128><<<sms * ctas, 128>>>(out, iters, bad);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    if (err == cudaSuccess) err = cudaGetLastError();
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long nb = 0;
    cudaMemcpy(&nb, bad, 8, cudaMemcpyDeviceToHost);
    // bytes stored + loaded per SM per cycle (at 1.965 GHz)
    const double bytes = 2.0 * ctas * 128.0 * 64 * 8 * iters;
    printf("%s{\"ctas_per_sm\": %d, \"status\": \"%s\", \"mismatches\": %llu, \"ms\": %.3f, "
           "\"st_plus_ld_bytes_per_clk_per_sm\": %.1f}",
           first ? "" : ", ", ctas, cudaGetErrorString(err), nb, ms, bytes / (ms * 1e-3 * 1.965e9));
    first = false;
  }
  printf("]}\n");
  return 0;
}
