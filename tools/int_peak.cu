// int_peak.cu — measured integer-ALU ceiling of the min-hash inner loop on
// this GPU (the roofline denominator of the hash stages).
//
// Each thread evaluates h = (A v + B) mod (2^31 - 1) (one 32x32->64 multiply
// add, the Mersenne fold and one conditional subtract, exactly the
// library's m31_hash) and keeps the running minimum, for 8 independent
// (A, B) chains over a register-generated stream of v: no memory traffic, so
// the rate is bounded only by the ALU / FMA pipes and issue.  Output: hash
// evaluations (entry x trial) per second at the clock the run saw, and the
// same rate x 7 (the instructions bench.py counts per (entry, trial)).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/int_peak tools/int_peak.cu
//   /tmp/int_peak > profiles/int_peak.json
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t m31_hash(uint32_t A, uint32_t B, uint32_t v) {
  uint64_t t = (uint64_t)A * v + B;
  uint32_t lo = (uint32_t)t & 0x7FFFFFFFu;
  uint32_t hi = (uint32_t)(t >> 31);
  uint32_t x = lo + hi;
  uint32_t y = x - 0x7FFFFFFFu;
  return x < y ? x : y;
}

constexpr int kChains = 8;

__global__ void __launch_bounds__(256) hash_peak(const uint32_t *AB, int iters, uint32_t *out) {
  uint32_t A[kChains], B[kChains], m[kChains];
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int c = 0; c < kChains; ++c) {
    A[c] = AB[(t + c) & 1023] | 1u;
    B[c] = AB[(t + 7 * c + 512) & 1023];
    m[c] = 0xFFFFFFFFu;
  }
  uint32_t v = t * 2654435761u;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < kChains; ++c) m[c] = min(m[c], m31_hash(A[c], B[c], v));
    v += 0x9E3779B9u;
  }
  uint32_t r = 0;
#pragma unroll
  for (int c = 0; c < kChains; ++c) r ^= m[c];
  out[t] = r;
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  uint32_t *ab, *out;
  cudaMalloc(&ab, 1024 * 4);
  uint32_t h[1024];
  uint64_t s = 12345;
  for (int i = 0; i < 1024; ++i) {
    s = s * 6364136223846793005ull + 1442695040888963407ull;
    h[i] = (uint32_t)(s >> 33) % 0x7FFFFFFFu;
  }
  cudaMemcpy(ab, h, sizeof h, cudaMemcpyHostToDevice);
  const int blocks = sms * 8, threads = 256, iters = 20000;
  cudaMalloc(&out, (size_t)blocks * threads * 4);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  hash_peak<<<blocks, threads>>>(ab, 100, out);   // warm-up
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0);
    hash_peak<<<blocks, threads>>>(ab, iters, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  const double evals = (double)blocks * threads * iters * kChains;
  const double rate = evals / (best / 1e3);
  printf("{\"hash_evals_per_s\": %.4e, \"hash_mix_tinstr_per_s\": %.3f, \"ms\": %.3f, \"sms\": %d, "
         "\"clock_mhz_attr\": %d, \"how\": \"tools/int_peak.cu: %d chains of m31_hash + min per thread, "
         "register-only, %d blocks x %d threads x %d iters, best of 5 (CUDA events); rate x 7 = the "
         "instructions bench.py counts per (entry, trial)\"}\n",
         rate, rate * 7 / 1e12, best, sms, clk / 1000, kChains, blocks, threads, iters);
  return 0;
}
