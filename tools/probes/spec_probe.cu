// Probe: per-step latency of the event engine's speculation-loop skeleton on one CTA (B200).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "../../paper_conf_date_shelm19_b200/csrc/snn_device.cuh"
using namespace snn;

template <int MODE>
__global__ void loop_kernel(int steps, const uint16_t* g_rows, const uint32_t* g_offs, unsigned long long* out, int ltd_lanes) {
  __shared__ uint32_t s_w[784 * 8];
  __shared__ uint16_t s_rows[4096];
  __shared__ uint32_t s_offs[1025];
  __shared__ int s_flag;
  for (int k = threadIdx.x; k < 784 * 8; k += blockDim.x) s_w[k] = k * 2654435761u;
  for (int k = threadIdx.x; k < 4096; k += blockDim.x) s_rows[k] = g_rows[k];
  for (int k = threadIdx.x; k <= 1024; k += blockDim.x) s_offs[k] = g_offs[k];
  if (threadIdx.x == 0) s_flag = 1 << 30;
  __syncthreads();
  const int tid = threadIdx.x, lane = tid & 31;
  const int wj = tid >> 2, f = tid & 3, fsh = f * 2, wpr = 8;
  const uint32_t* wcol = s_w + (wj & 7);
  float v[4] = {-70.f, -70.f, -70.f, -70.f};
  const uint32_t flag_addr = smem_u32(&s_flag);
  bool done = false;
  int kk = 0;
  int r0 = s_offs[0];
  const bool ltd_me = lane < ltd_lanes;
  unsigned long long t0 = clock64();
  uint32_t evsum = 0;
  while (MODE == 0 ? kk < steps : __any_sync(FULL, !done)) {
    if (!done && (kk >= steps || kk > ld_volatile_shared_u32addr(flag_addr))) { done = true; }
    if (kk >= steps) break;
    const int r1 = s_offs[(kk & 1023) + 1];
    if (!done) {
      uint32_t acc = 0;
      int r = r0;
      for (; r + 4 <= r1; r += 4) {
        const int i0 = s_rows[r], i1 = s_rows[r + 1], i2 = s_rows[r + 2], i3 = s_rows[r + 3];
        acc += ((wcol[i0 * wpr] >> fsh) & 0x03030303u) + ((wcol[i1 * wpr] >> fsh) & 0x03030303u) +
               ((wcol[i2 * wpr] >> fsh) & 0x03030303u) + ((wcol[i3 * wpr] >> fsh) & 0x03030303u);
      }
      for (; r < r1; ++r) acc += (wcol[(int)s_rows[r] * wpr] >> fsh) & 0x03030303u;
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const float I = __fmul_rn(__int2float_rn((acc >> (8 * c)) & 0xFF), 0.5f);
        const float y = __fmaf_rn(0.314f, I, -6.77f);
        const float dv = __fmaf_rn(-0.0989f, v[c], y);
        v[c] = __fmaf_rn(1.0f, dv, v[c]);
        if (v[c] > 10000.f) done = true;
      }
    }
    if (MODE >= 2) {
      const bool ltd_on = MODE == 3 && ltd_me && !done;
      if (__any_sync(FULL, ltd_on)) {
#pragma unroll 1
        for (uint32_t lm = __ballot_sync(FULL, ltd_on); lm; lm &= lm - 1) {
          const int Ls = __ffs(lm) - 1;
#pragma unroll 1
          for (int c0 = r0; c0 < r1; c0 += 32) {
            const int n = min(32, r1 - c0);
            bool bit = false;
            if (lane < n) {
              const uint4 u = philox((uint32_t)kk, (uint32_t)s_rows[c0 + lane], (uint32_t)(Ls >> 2), TAG_LTD, 12345ull);
              bit = pick(u, Ls & 3) <= 0x10000000u;
            }
            const uint32_t m = __ballot_sync(FULL, bit);
            if (lane == Ls) evsum += __popc(m);
          }
        }
      }
    }
    ++kk;
    r0 = r1;
  }
  unsigned long long t1 = clock64();
  if (lane == 0) out[blockIdx.x * 32 + (tid >> 5)] = t1 - t0;
  if (v[0] == 1.2345f && evsum == 7) out[1023] = 1;
}

int main() {
  const int steps = 1000;
  // rows: 6 per step, spread across 784 inputs
  uint16_t h_rows[4096]; uint32_t h_offs[1025];
  for (int k = 0; k <= 1024; ++k) h_offs[k] = (k * 6) % 4096 < (k * 6) ? 0 : k * 6;
  for (int k = 0; k <= 1024; ++k) h_offs[k] = (uint32_t)(k < 682 ? k * 6 : 4092);
  for (int r = 0; r < 4096; ++r) h_rows[r] = (uint16_t)((r * 131) % 784);
  uint16_t* d_rows; uint32_t* d_offs; unsigned long long* d_out;
  cudaMalloc(&d_rows, sizeof(h_rows)); cudaMalloc(&d_offs, sizeof(h_offs)); cudaMalloc(&d_out, 1024 * 8);
  cudaMemcpy(d_rows, h_rows, sizeof(h_rows), cudaMemcpyHostToDevice);
  cudaMemcpy(d_offs, h_offs, sizeof(h_offs), cudaMemcpyHostToDevice);
  unsigned long long h_out[1024];
  auto run = [&](auto kern, const char* name, int threads, int ltd) {
    kern<<<1, threads>>>(600, d_rows, d_offs, d_out, ltd);
    cudaDeviceSynchronize();
    cudaMemset(d_out, 0, 1024 * 8);
    kern<<<1, threads>>>(600, d_rows, d_offs, d_out, ltd);
    cudaDeviceSynchronize();
    cudaMemcpy(h_out, d_out, 1024 * 8, cudaMemcpyDeviceToHost);
    unsigned long long mx = 0; for (int w = 0; w < threads / 32; ++w) mx = h_out[w] > mx ? h_out[w] : mx;
    printf("%-40s threads=%4d ltd_lanes=%2d: %7.1f cycles/step (%s)\n", name, threads, ltd, mx / 600.0, cudaGetErrorString(cudaGetLastError()));
  };
  for (int threads : {32, 128, 256, 512}) {
    run(loop_kernel<0>, "A: flag+offs+integrate+LIF", threads, 0);
    run(loop_kernel<1>, "B: A + __any_sync loop", threads, 0);
    run(loop_kernel<2>, "C: B + idle LTD ballot", threads, 0);
    run(loop_kernel<3>, "D: C + 1 LTD lane/warp", threads, 1);
    run(loop_kernel<3>, "D: C + 4 LTD lanes/warp", threads, 4);
  }
  return 0;
}
