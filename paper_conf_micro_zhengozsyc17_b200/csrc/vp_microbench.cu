// vp_microbench.cu — measured ceilings for the rooflines that have no datasheet number
// (SURVEY §8(d) "L2 atomics: measured by a microbenchmark").
//
// vp_bench_red_min_u64: fire-and-forget 64-bit atomic minimum (RED.MIN.U64, the raster
// z-buffer update of reading R-S6) from every thread of a full grid to pseudo-random
// 8-B slots of a `slots`-entry buffer (16.6 MB at 1920x1080 fits the 126 MB L2), timed
// with CUDA events on the default stream.  Returns the L2 atomic rate the Fragment
// stage's roofline is quoted against.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/vp.h"

namespace {

__global__ void k_red_min(unsigned long long* buf, unsigned long long slots, unsigned long long per_thread,
                          unsigned long long seed) {
  const unsigned long long tid = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
  unsigned long long x = seed ^ (tid * 0x9E3779B97F4A7C15ull);
  for (unsigned long long i = 0; i < per_thread; ++i) {
    x ^= x << 13;
    x ^= x >> 7;
    x ^= x << 17;
    atomicMin(buf + (x % slots), x);  // result unused: compiled to RED.E.MIN.64
  }
}
__global__ void k_fill(unsigned long long* buf, unsigned long long n) {
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    buf[i] = ~0ull;
}

}  // namespace

extern "C" vp_status vp_bench_red_min_u64(int device, unsigned long long slots, unsigned long long n_ops,
                                          double* ops_per_s) {
  if (!ops_per_s || slots == 0 || n_ops == 0) return VP_ERR_INVALID;
  int prev = 0;
  cudaGetDevice(&prev);
  if (cudaSetDevice(device) != cudaSuccess) return VP_ERR_CUDA;
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, device);
  const int blocks = prop.multiProcessorCount * 8, threads = 256;
  const unsigned long long per = (n_ops + (unsigned long long)blocks * threads - 1) / ((unsigned long long)blocks * threads);
  unsigned long long* buf = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  vp_status rc = VP_OK;
  if (cudaMalloc(&buf, slots * 8) != cudaSuccess) rc = VP_ERR_OOM;
  if (rc == VP_OK && (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess)) rc = VP_ERR_CUDA;
  if (rc == VP_OK) {
    k_fill<<<blocks, threads>>>(buf, slots);
    k_red_min<<<blocks, threads>>>(buf, slots, per, 1);  // warm-up (L2 residency)
    float best = 1e30f;
    for (int r = 0; r < 3; ++r) {
      cudaEventRecord(e0);
      k_red_min<<<blocks, threads>>>(buf, slots, per, 2 + r);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0.f;
      cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    if (cudaGetLastError() != cudaSuccess) rc = VP_ERR_CUDA;
    *ops_per_s = (double)per * blocks * threads / (best * 1e-3);
  }
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  cudaFree(buf);
  cudaSetDevice(prev);
  return rc;
}
