// microbench.cu -- measure the sync primitives the persistent kernels rely on
// (B200): __nanosleep granularity and the SM-to-SM flag ping-pong latency
// through L2 with relaxed and release/acquire accesses.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu && /tmp/mb
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned ldr(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void str(unsigned* p, unsigned v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__global__ void sleep_k(unsigned ns, unsigned long long* out) {
  unsigned long long t0 = gt();
  for (int i = 0; i < 100; ++i) __nanosleep(ns);
  out[0] = (gt() - t0) / 100;
}

// two CTAs bounce a counter `iters` times; sleep_ns > 0 adds a backoff in the spin
__global__ void pingpong(unsigned* flag, int iters, unsigned sleep_ns, unsigned long long* out) {
  if (threadIdx.x != 0) return;
  const unsigned me = blockIdx.x;   // 0 or 1
  unsigned long long t0 = gt();
  for (int i = 0; i < iters; ++i) {
    const unsigned want = 2 * i + me;
    while (ldr(flag) != want) {
      if (sleep_ns) __nanosleep(sleep_ns);
    }
    str(flag, want + 1);
  }
  if (me == 0) out[0] = (gt() - t0) / (2 * iters);   // one-way latency
}

// ping-pong between blocks 0/1 while every other block's threads spin on
// never-ready words (as waiting consumers do), sleeping sleep_ns per poll
__global__ void pingpong_loaded(unsigned* flag, const unsigned long long* junk, int iters, unsigned sleep_ns,
                                unsigned long long* out, unsigned* stop) {
  if (blockIdx.x >= 2) {
    const unsigned long long* p = junk + (size_t(blockIdx.x) * blockDim.x + threadIdx.x) * 4;
    unsigned long long acc = 0;
    while (true) {
      unsigned long long a, b;
      asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
      acc += a ^ b;
      if (ldr(stop)) break;
      __nanosleep(sleep_ns);
    }
    if (acc == 12345) out[1] = acc;
    return;
  }
  if (threadIdx.x != 0) return;
  const unsigned me = blockIdx.x;
  unsigned long long t0 = gt();
  for (int i = 0; i < iters; ++i) {
    const unsigned want = 2 * i + me;
    while (ldr(flag) != want) {
    }
    str(flag, want + 1);
  }
  if (me == 0) {
    out[0] = (gt() - t0) / (2 * iters);
    str(stop, 1);
  }
}

// clock64 cost of a dependent L2 load chain (pointer chase on a tiny buffer)
__global__ void chase(const unsigned* buf, int iters, unsigned long long* out) {
  unsigned j = 0;
  unsigned long long t0 = gt();
  for (int i = 0; i < iters; ++i) j = ldr(buf + j);
  out[0] = (gt() - t0) / iters;
  out[1] = j;
}

int main() {
  unsigned long long* d_out;
  unsigned* flag;
  unsigned* buf;
  cudaMalloc(&d_out, 64);
  cudaMalloc(&flag, 4);
  cudaMalloc(&buf, 1 << 20);
  unsigned long long h[2];
  for (unsigned ns : {0u, 20u, 100u, 500u, 1000u}) {
    sleep_k<<<1, 32>>>(ns, d_out);
    cudaMemcpy(h, d_out, 8, cudaMemcpyDeviceToHost);
    printf("nanosleep(%u): %llu ns per call\n", ns, h[0]);
  }
  for (unsigned ns : {0u, 20u, 100u}) {
    cudaMemset(flag, 0, 4);
    pingpong<<<2, 32>>>(flag, 2000, ns, d_out);
    cudaMemcpy(h, d_out, 8, cudaMemcpyDeviceToHost);
    printf("ping-pong one-way latency, spin sleep %u ns: %llu ns\n", ns, h[0]);
  }
  {
    unsigned long long* junk;
    unsigned* stop;
    cudaMalloc(&junk, size_t(148) * 512 * 32 + 64);
    cudaMemset(junk, 0, size_t(148) * 512 * 32 + 64);
    cudaMalloc(&stop, 4);
    for (unsigned ns : {20u, 100u, 500u}) {
      cudaMemset(flag, 0, 4);
      cudaMemset(stop, 0, 4);
      pingpong_loaded<<<148, 512>>>(flag, junk, 2000, ns, d_out, stop);
      cudaMemcpy(h, d_out, 8, cudaMemcpyDeviceToHost);
      printf("ping-pong one-way latency with 146x512 pollers (sleep %u ns): %llu ns\n", ns, h[0]);
    }
  }
  // pointer chase: buf[j] = (j + 32) mod 4096 (stays in L2 after first touch)
  unsigned hb[4096];
  for (int i = 0; i < 4096; ++i) hb[i] = (i + 32) % 4096;
  cudaMemcpy(buf, hb, sizeof hb, cudaMemcpyHostToDevice);
  chase<<<1, 1>>>(buf, 10000, d_out);
  cudaMemcpy(h, d_out, 16, cudaMemcpyDeviceToHost);
  printf("dependent relaxed.gpu load (L2 hit): %llu ns\n", h[0]);
  printf("err: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
