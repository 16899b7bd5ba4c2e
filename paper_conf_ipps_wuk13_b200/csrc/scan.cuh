// scan.cuh — block-level and small device-wide exclusive scans (hand-written;
// no CUB / Thrust on the path).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace sg {

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T u = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += u;
  }
  return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Exclusive scan across the block (blockDim.x multiple of 32, <= 1024).
// `ws` is shared scratch of >= 33 elements.  Returns the exclusive prefix and
// writes the block total to *total (all threads).  Contains __syncthreads.
template <typename T>
__device__ __forceinline__ T block_excl_scan(T v, T *ws, T *total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int nw = blockDim.x >> 5;
  T inc = warp_incl_scan(v);
  if (lane == 31) ws[wid] = inc;
  __syncthreads();
  if (wid == 0) {
    T x = lane < nw ? ws[lane] : T(0);
    T xi = warp_incl_scan(x);
    if (lane < nw) ws[lane] = xi - x;
    if (lane == 31) ws[32] = xi;
  }
  __syncthreads();
  T r = ws[wid] + inc - v;
  *total = ws[32];
  __syncthreads();
  return r;
}

}  // namespace sg
