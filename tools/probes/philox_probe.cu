// Latency/throughput probe of the device Philox4x32-10 (snn_device.cuh) inside one CTA of 224 threads:
// cycles for K independent Philox blocks per thread, all 7 warps at once (the lean kernel's winner-CTA phase).
#include <cstdio>
#include "../../paper_conf_date_shelm19_b200/csrc/snn_device.cuh"
using namespace snn;
template <int K>
__global__ void probe(unsigned long long* out, unsigned long long seed, uint32_t* sink) {
  __syncthreads();
  const long long t0 = clock64();
  uint32_t acc = 0;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint4 u = philox((uint32_t)(threadIdx.x + 7 * k), (uint32_t)k, 11u, 2u, seed);
    acc ^= u.x ^ u.y ^ u.z ^ u.w;
  }
  const long long t1 = clock64();
  sink[threadIdx.x] = acc;
  if (threadIdx.x == 0) out[K] = (unsigned long long)(t1 - t0);
}
int main() {
  unsigned long long* d;
  uint32_t* s;
  cudaMalloc(&d, 64 * 8);
  cudaMalloc(&s, 1024 * 4);
  for (int it = 0; it < 3; ++it) {
    probe<1><<<1, 224>>>(d, 5, s);
    probe<2><<<1, 224>>>(d, 5, s);
    probe<3><<<1, 224>>>(d, 5, s);
    probe<4><<<1, 224>>>(d, 5, s);
    probe<8><<<1, 224>>>(d, 5, s);
  }
  unsigned long long h[64] = {0};
  cudaMemcpy(h, d, 64 * 8, cudaMemcpyDeviceToHost);
  for (int k : {1, 2, 3, 4, 8}) printf("224 threads, %d Philox4x32-10 per thread: %llu cycles (thread 0)\n", k, h[k]);
  probe<1><<<1, 32>>>(d, 5, s);
  cudaMemcpy(h, d, 64 * 8, cudaMemcpyDeviceToHost);
  printf("32 threads, 1 Philox per thread: %llu cycles\n", h[1]);
  return 0;
}
