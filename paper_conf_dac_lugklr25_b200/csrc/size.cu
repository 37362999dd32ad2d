// size.cu -- device steps of INSTA-Size: the
// stage gradients ("the gradient sum of a cell arc and its driving net arc")
// and the threshold + rank selection of critical stages.  The sizing loop
// around them (candidate table, 3-hop blocking, commit / rollback on TNS) is
// host orchestration over the C ABI (paper_conf_dac_lugklr25_b200/size.py).
#include <cuda_runtime.h>

#include <cub/cub.cuh>

#include <algorithm>
#include <cstdint>

#include "device_common.cuh"
#include "internal.h"

namespace insta {

// a thread per fanin position q: stage gradient of the arc at q (caller order)
__global__ void stage_grad_kernel(int64_t e, const int32_t* __restrict__ fanin_ptr, const int32_t* __restrict__ fin_src,
                                  const int32_t* __restrict__ fin_arc, const uint8_t* __restrict__ arc_class,
                                  const float2* __restrict__ d_mean, float* out) {
  const long long q = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (q >= e) return;
  const int arc = __ldg(fin_arc + q);
  if (__ldg(arc_class + arc) != 1) {
    out[arc] = 0.f;
    return;
  }
  const float2 dc = d_mean[arc];
  float s = dc.x + dc.y;
  const int p = __ldg(fin_src + q) & kSrcMask;   // the cell's input pin
  const int b0 = __ldg(fanin_ptr + p), b1 = __ldg(fanin_ptr + p + 1);
  if (b1 - b0 == 1) {
    const int an = __ldg(fin_arc + b0);
    if (__ldg(arc_class + an) == 0) {
      const float2 dn = d_mean[an];
      s += dn.x + dn.y;
    }
  }
  out[arc] = s;
}

struct BelowThreshold {
  const float* grad;
  float thr;
  __device__ __forceinline__ bool operator()(const int32_t& a) const { return grad[a] < -thr; }
};

__global__ void iota_kernel(int64_t n, int32_t* out) {
  const long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (k < n) out[k] = int32_t(k);
}

// keys of the selected ids; the unused tail gets +inf (sorts behind them)
__global__ void gather_keys_kernel(int n, const int32_t* __restrict__ count, int32_t* idx,
                                   const float* __restrict__ grad, float* keys) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  if (k < *count) {
    keys[k] = grad[idx[k]];
  } else {
    keys[k] = __int_as_float(0x7f800000);
    idx[k] = -1;
  }
}

int launch_stage_gradients(DevGraph& g, const float* d_mean, float* out, void* stream) {
  if (g.e == 0) return 0;
  stage_grad_kernel<<<unsigned((g.e + 255) / 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
      g.e, g.fanin_ptr, g.fin_src, g.fin_arc, g.arc_class, reinterpret_cast<const float2*>(d_mean), out);
  return int(cudaGetLastError());
}

// stages with grad < -threshold, most negative first (stable: ties by arc id);
// out_arcs DEVICE int32[num_arcs], out_count DEVICE int32[1]
int launch_select_stages(DevGraph& g, const float* grad, float threshold, int32_t* out_arcs, int32_t* out_count,
                         void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int64_t n = g.e;
  if (n == 0) return int(cudaMemsetAsync(out_count, 0, sizeof(int32_t), st));
  if (n >= (int64_t(1) << 31)) return int(cudaErrorInvalidValue);
  const int ni = int(n);
  // scratch: ids, selected ids, keys, sorted keys + CUB temp storage
  size_t t_sel = 0, t_sort = 0;
  BelowThreshold pred{grad, threshold};
  cub::DeviceSelect::If(nullptr, t_sel, (int32_t*)nullptr, (int32_t*)nullptr, (int32_t*)nullptr, ni, pred, st);
  cub::DeviceRadixSort::SortPairs(nullptr, t_sort, (float*)nullptr, (float*)nullptr, (int32_t*)nullptr,
                                  (int32_t*)nullptr, ni, 0, 32, st);
  const size_t need = size_t(ni) * 4 * 4 + std::max(t_sel, t_sort) + 256;
  if (g.sz_cap < need) {
    if (g.sz_tmp) cudaFree(g.sz_tmp);
    g.sz_tmp = nullptr;
    cudaError_t e = cudaMalloc(&g.sz_tmp, need);
    if (e != cudaSuccess) return int(e);
    g.sz_cap = need;
  }
  char* base = static_cast<char*>(g.sz_tmp);
  int32_t* ids = reinterpret_cast<int32_t*>(base);
  int32_t* sel = ids + ni;
  float* keys = reinterpret_cast<float*>(sel + ni);
  float* keys_out = keys + ni;
  void* tmp = keys_out + ni;
  iota_kernel<<<unsigned((n + 255) / 256), 256, 0, st>>>(n, ids);
  size_t t = t_sel;
  cudaError_t e = cub::DeviceSelect::If(tmp, t, ids, sel, out_count, ni, pred, st);
  if (e != cudaSuccess) return int(e);
  gather_keys_kernel<<<unsigned((n + 255) / 256), 256, 0, st>>>(ni, out_count, sel, grad, keys);
  t = t_sort;   // radix sort is stable: equal gradients keep arc id order
  e = cub::DeviceRadixSort::SortPairs(tmp, t, keys, keys_out, sel, out_arcs, ni, 0, 32, st);
  return int(e != cudaSuccess ? e : cudaGetLastError());
}

}  // namespace insta
