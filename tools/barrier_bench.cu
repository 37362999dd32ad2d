// Grid-barrier latency on the B200 (148 CTAs, one per SM): variants of the
// sweep's per-level barrier.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/barrier_bench.cu -o /tmp/bb
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

template <int V>
__global__ void bar_kernel(unsigned* ctr, int iters, unsigned long long* out) {
  unsigned long long t0 = 0;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t0));
  for (int k = 1; k <= iters; ++k) {
    if (V == 3) {
      cg::this_grid().sync();
      continue;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      const unsigned target = k * gridDim.x;
      if (V == 0) {
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
        unsigned v;
        do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory"); } while (v < target);
      } else if (V == 1) {
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
        unsigned v;
        do { asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory"); } while (v < target);
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      } else if (V == 2) {
        unsigned v;
        asm volatile("atom.add.release.gpu.global.u32 %0, [%1], 1;" : "=r"(v) : "l"(ctr) : "memory");
        while (v + 1 < target && true) {
          asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
          if (v >= target) break;
          v = v;
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
    }
    __syncthreads();
  }
  unsigned long long t1;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t1));
  if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = t1 - t0;
}

template <int V>
void run(const char* name, int threads) {
  unsigned* ctr;
  unsigned long long* out;
  cudaMalloc(&ctr, 4);
  cudaMalloc(&out, 8);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int iters = 1000;
  for (int rep = 0; rep < 3; ++rep) {
    cudaMemset(ctr, 0, 4);
    void* args[] = {&ctr, &iters, &out};
    cudaLaunchCooperativeKernel((void*)bar_kernel<V>, sms, threads, args, 0, 0);
    cudaDeviceSynchronize();
    unsigned long long t;
    cudaMemcpy(&t, out, 8, cudaMemcpyDeviceToHost);
    printf("%-28s threads %4d: %.3f us per barrier (%s)\n", name, threads, t / 1e3 / iters,
           cudaGetErrorString(cudaGetLastError()));
  }
}

int main() {
  for (int th : {384, 1024}) {
    run<0>("red.release + ld.acquire", th);
    run<1>("red.release + ld.relaxed", th);
    run<2>("atom.release + ld.relaxed", th);
    run<3>("cg grid.sync", th);
  }
  return 0;
}
