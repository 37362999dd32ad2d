// Latency of dependent FP64 / conversion / sqrt chains on this GPU (cycles per op).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(double* out, float* outf, long long* cyc, int n, double a, float b) {
  double x = a;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) x = x + a;           // DADD chain
  long long t1 = clock64();
  for (int i = 0; i < n; ++i) x = x * 1.0000001;   // DMUL chain
  long long t2 = clock64();
  float f = b;
  for (int i = 0; i < n; ++i) f = float(double(f) + 1.0);   // F2F + DADD + F2F chain
  long long t3 = clock64();
  float y = b;
  for (int i = 0; i < n; ++i) y = sqrtf(y + 2.0f);  // IEEE sqrtf chain
  long long t4 = clock64();
  float z = b;
  for (int i = 0; i < n; ++i) z = z * 1.0001f + 0.5f;   // FMUL+FADD chain
  long long t5 = clock64();
  out[0] = x; outf[0] = f + y + z;
  cyc[0] = (t1 - t0) / n; cyc[1] = (t2 - t1) / n; cyc[2] = (t3 - t2) / n; cyc[3] = (t4 - t3) / n; cyc[4] = (t5 - t4) / n;
}
int main() {
  double* o; float* of; long long* c; cudaMalloc(&o, 8); cudaMalloc(&of, 4); cudaMalloc(&c, 64);
  k<<<1, 1>>>(o, of, c, 10000, 1.0, 2.0f);
  long long h[5]; cudaMemcpy(h, c, 40, cudaMemcpyDeviceToHost);
  printf("cycles per op: DADD %lld, DMUL %lld, F2F+DADD+F2F %lld, sqrtf+FADD %lld, FMUL+FADD %lld\n", h[0], h[1], h[2], h[3], h[4]);
  return 0;
}
