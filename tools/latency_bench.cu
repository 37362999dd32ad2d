// Dependent global-load latency after a grid barrier (sweep cone-pass pattern):
// per iteration, a barrier then a chain of D dependent random loads per thread.
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void gsync(unsigned* ctr, unsigned target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
    unsigned v;
    do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory"); } while (v < target);
  }
  __syncthreads();
}

template <int MODE>
__global__ void lat_kernel(unsigned* ctr, const unsigned* __restrict__ a, unsigned mask, int iters, int depth,
                           unsigned long long* out, unsigned* sink) {
  unsigned long long t0;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t0));
  unsigned x = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u;
  for (int k = 1; k <= iters; ++k) {
    gsync(ctr, k * gridDim.x);
    for (int d = 0; d < depth; ++d) {
      unsigned v;
      const unsigned* p = a + ((x * 2654435761u) & mask);
      if (MODE == 0) asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p));
      else if (MODE == 1) v = __ldcg(p);
      else v = __ldg(p);
      x += v;
    }
  }
  unsigned long long t1;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t1));
  if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = t1 - t0;
  if (x == 0x12345) sink[0] = x;
}

int main() {
  unsigned *ctr, *a, *sink;
  unsigned long long* out;
  const size_t n = 1 << 24;   // 64 MB
  cudaMalloc(&ctr, 4);
  cudaMalloc(&a, n * 4);
  cudaMemset(a, 0, n * 4);
  cudaMalloc(&sink, 4);
  cudaMalloc(&out, 8);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const char* names[] = {"ld.relaxed.gpu", "ld.global.cg", "ld.global.nc"};
  for (int mode = 0; mode < 3; ++mode) {
    for (int depth : {0, 1, 2, 4}) {
      for (int threads : {64, 384}) {
        unsigned mask = unsigned(n - 1);
        int iters = 200;
        cudaMemset(ctr, 0, 4);
        void* args[] = {&ctr, &a, &mask, &iters, &depth, &out, &sink};
        void* fn = mode == 0 ? (void*)lat_kernel<0> : mode == 1 ? (void*)lat_kernel<1> : (void*)lat_kernel<2>;
        cudaLaunchCooperativeKernel(fn, sms, threads, args, 0, 0);
        cudaDeviceSynchronize();
        unsigned long long t;
        cudaMemcpy(&t, out, 8, cudaMemcpyDeviceToHost);
        printf("%-16s depth %d threads %3d: %.3f us per iteration (%s)\n", names[mode], depth, threads,
               t / 1e3 / iters, cudaGetErrorString(cudaGetLastError()));
      }
    }
  }
  return 0;
}
