// Microbenchmark / probe (not on the product path): are conflicting
// shared-memory atomicAdds of ONE warp instruction resolved in lane order?
// Every warp repeatedly adds 1 to counters chosen by a hash of (lane, iter)
// (few addresses -> many conflicts) and checks that, among the lanes that hit
// the same counter, the returned old values increase with the lane index.
// Prints the number of warp-instructions where that order was violated.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/atom_order tools/atom_order.cu
#include <cstdio>
#include <cstdint>

__global__ void probe(unsigned long long *viol, unsigned long long *total, int iters, int naddr, int packed) {
  __shared__ uint32_t ctr[8][1024];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = lane; i < 1024; i += 32) ctr[w][i] = 0;
  __syncwarp();
  unsigned long long v = 0;
  for (int it = 0; it < iters; ++it) {
    uint32_t h = (uint32_t)(lane * 2654435761u) ^ (uint32_t)(it * 0x9E3779B9u) ^ (blockIdx.x * 77u);
    h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
    const uint32_t a = h % (uint32_t)naddr;
    uint32_t old;
    if (packed) old = atomicAdd(&ctr[w][a >> 1], 1u << ((a & 1) * 16)) >> ((a & 1) * 16) & 0xFFFFu;
    else old = atomicAdd(&ctr[w][a], 1u);
    // peers with the same address and a lower lane must have smaller olds
    const uint32_t m = __match_any_sync(0xffffffffu, a);
    uint32_t lower = m & ((1u << lane) - 1u);
    bool bad = false;
    for (int l = 0; l < 32; ++l) {
      const uint32_t o2 = __shfl_sync(0xffffffffu, old, l);
      if ((lower >> l) & 1u) bad |= o2 > old;
    }
    if (__any_sync(0xffffffffu, bad) && lane == 0) ++v;
    if ((it & 1023) == 1023) {                   // keep packed counters below 2^16
      __syncwarp();
      for (int i = lane; i < 1024; i += 32) ctr[w][i] = 0;
      __syncwarp();
    }
  }
  if (lane == 0) {
    atomicAdd(viol, v);
    atomicAdd(total, (unsigned long long)iters);
  }
}

int main() {
  unsigned long long *d;
  cudaMalloc(&d, 16);
  for (int packed = 0; packed < 2; ++packed)
    for (int naddr : {2, 8, 64, 1024}) {
      cudaMemset(d, 0, 16);
      probe<<<148 * 4, 256>>>(d, d + 1, 4096, naddr, packed);
      unsigned long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      printf("{\"packed\": %d, \"naddr\": %d, \"warp_instructions\": %llu, \"out_of_lane_order\": %llu}\n",
             packed, naddr, h[1], h[0]);
    }
  return 0;
}
