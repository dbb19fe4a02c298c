// tma_probe.cu -- minimal checks of fp64 TMA tile loads (debugging aid for
// the phi-sweep staging): descriptor as __grid_constant__, in global memory,
// and box shapes.  nvcc -gencode arch=compute_100a,code=sm_100a -o tma_probe tools/tma_probe.cu
#include <cstdio>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>

struct alignas(64) Desc { unsigned long long v[16]; };

__device__ __forceinline__ unsigned s32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ void load(const void* dptr, double* buf, unsigned long long* bar, int rank, int bx, int by, int bz,
                     unsigned bytes) {
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(s32(bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(s32(bar)), "r"(bytes) : "memory");
    if (rank == 4)
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];\n"
                   ::"r"(s32(buf)), "l"(dptr), "r"(bx), "r"(by), "r"(bz), "r"(0), "r"(s32(bar)) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n"
                   ::"r"(s32(buf)), "l"(dptr), "r"(bx), "r"(by), "r"(s32(bar)) : "memory");
  }
  asm volatile("{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W_%=;\n}\n" ::"r"(s32(bar)) : "memory");
}

__global__ void k_bulk(const double* src, double* out, unsigned bytes) {
  __shared__ __align__(128) double buf[34 * 10 * 4];
  __shared__ __align__(8) unsigned long long bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(s32(&bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(s32(&bar)), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n"
                 ::"r"(s32(buf)), "l"(src), "r"(bytes), "r"(s32(&bar)) : "memory");
  }
  asm volatile("{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W_%=;\n}\n" ::"r"(s32(&bar)) : "memory");
  for (int i = threadIdx.x; i < (int)(bytes / 8); i += blockDim.x) out[i] = buf[i];
}

__global__ void k_param(const __grid_constant__ Desc d, double* out, int rank, unsigned bytes) {
  __shared__ __align__(128) double buf[34 * 10 * 4];
  __shared__ __align__(8) unsigned long long bar;
  load(&d, buf, &bar, rank, 15, 1, 3, bytes);
  for (int i = threadIdx.x; i < (int)(bytes / 8); i += blockDim.x) out[i] = buf[i];
}
__global__ void k_global(const Desc* d, double* out, int rank, unsigned bytes) {
  __shared__ __align__(128) double buf[34 * 10 * 4];
  __shared__ __align__(8) unsigned long long bar;
  asm volatile("fence.proxy.tensormap::generic.acquire.gpu [%0], 128;\n" ::"l"(d) : "memory");
  load(d, buf, &bar, rank, 15, 1, 3, bytes);
  for (int i = threadIdx.x; i < (int)(bytes / 8); i += blockDim.x) out[i] = buf[i];
}

int main(int argc, char** argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;  // 0: bulk 1-D, 1: param 2-D, 2: global 2-D, 3: param 4-D, 4: global 4-D
  const int pitch = 64, ny = 20, nz = 20, nc = 4;
  const size_t n = (size_t)pitch * ny * nz * nc;
  double* h = new double[n];
  for (size_t i = 0; i < n; ++i) h[i] = (double)i;
  double *dg, *dout;
  Desc* ddesc;
  cudaMalloc(&dg, n * 8);
  cudaMalloc(&dout, 34 * 10 * 4 * 8);
  cudaMalloc(&ddesc, sizeof(Desc));
  cudaMemcpy(dg, h, n * 8, cudaMemcpyHostToDevice);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = (decltype(&cuTensorMapEncodeTiled))fn;
  if (mode == 0) {
    k_bulk<<<1, 128>>>(dg + 16, dout, 288);
    cudaError_t e = cudaDeviceSynchronize();
    double o[36];
    cudaMemcpy(o, dout, sizeof o, cudaMemcpyDeviceToHost);
    printf("bulk 1-D: %s  first %g last %g\n", cudaGetErrorString(e), o[0], o[35]);
    return e != cudaSuccess;
  }
  for (int rank : {2, 4}) {
    for (int where = 0; where < 2; ++where) {
      if (mode != (rank == 2 ? 1 : 3) + where) continue;
      Desc d;
      cuuint64_t dims[4] = {(cuuint64_t)pitch, (cuuint64_t)ny, (cuuint64_t)nz, (cuuint64_t)nc};
      cuuint64_t str[3] = {(cuuint64_t)pitch * 8, (cuuint64_t)pitch * ny * 8, (cuuint64_t)pitch * ny * nz * 8};
      cuuint32_t box[4] = {34, 10, 1, 4}, es[4] = {1, 1, 1, 1};
      if (rank == 2) dims[1] = (cuuint64_t)ny * nz * nc;
      CUresult r = enc((CUtensorMap*)&d, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, rank, dg, dims, str, box, es,
                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      unsigned bytes = rank == 4 ? 34 * 10 * 4 * 8 : 34 * 10 * 8;
      if (where == 0) k_param<<<1, 128>>>(d, dout, rank, bytes);
      else {
        cudaMemcpy(ddesc, &d, sizeof d, cudaMemcpyHostToDevice);
        k_global<<<1, 128>>>(ddesc, dout, rank, bytes);
      }
      cudaError_t e = cudaDeviceSynchronize();
      printf("rank %d where %s encode %d: %s\n", rank, where ? "global" : "param", (int)r, cudaGetErrorString(e));
      if (e != cudaSuccess) return 1;
    }
  }
  return 0;
}
