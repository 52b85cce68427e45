// Probe: cost per step of the event engine's block integration on B200 (one CTA).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void integ(int nsteps, const uint32_t* g_offs, const uint32_t* g_woff, unsigned long long* out, int* sink) {
  __shared__ uint32_t s_w[785 * 8];
  __shared__ uint32_t s_woff[2048];
  __shared__ uint32_t s_offs[1025];
  __shared__ uint32_t s_acc[8 * 256];
  for (int k = threadIdx.x; k < 785 * 8; k += blockDim.x) s_w[k] = k * 2654435761u;
  for (int k = threadIdx.x; k < 2048; k += blockDim.x) s_woff[k] = g_woff[k];
  for (int k = threadIdx.x; k <= 1024; k += blockDim.x) s_offs[k] = g_offs[k];
  __syncthreads();
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int TPW = 4, wj = tid / TPW, f = tid % TPW, fsh = f * 2;
  const uint32_t* wcol = s_w + (wj % 8);
  uint32_t* my_acc = s_acc + tid;
  const uint32_t LMASK = 0x03030303u;
  long long t0 = clock64();
  uint32_t total = 0;
  for (int kk0 = 0; kk0 + 8 <= nsteps; kk0 += 8) {
    int rb[9];
#pragma unroll
    for (int b = 0; b <= 8; ++b) rb[b] = s_offs[kk0 + b];
    if (MODE == 0) {            // as in the kernel: rolled over steps, unroll-4 rows + remainder
#pragma unroll 1
      for (int b = 0; b < 8; ++b) {
        const int ra = rb[b], re = rb[b + 1];
        uint32_t a0 = 0u, a1 = 0u;
        int r = ra;
        for (; r + 4 <= re; r += 4) {
          const uint32_t o0 = s_woff[r], o1 = s_woff[r + 1], o2 = s_woff[r + 2], o3 = s_woff[r + 3];
          a0 += ((wcol[o0] >> fsh) & LMASK) + ((wcol[o1] >> fsh) & LMASK);
          a1 += ((wcol[o2] >> fsh) & LMASK) + ((wcol[o3] >> fsh) & LMASK);
        }
        for (; r < re; ++r) a0 += (wcol[s_woff[r]] >> fsh) & LMASK;
        my_acc[b * nthr] = a0 + a1;
      }
    } else if (MODE == 1) {     // predicated, fully unrolled: 12 row slots per step, all 8 steps
#pragma unroll
      for (int b = 0; b < 8; ++b) {
        const int ra = rb[b], n = rb[b + 1] - rb[b];
        uint32_t a = 0u;
#pragma unroll
        for (int x = 0; x < 12; ++x) {
          const uint32_t o = s_woff[ra + x];
          const uint32_t w = wcol[o];
          a += (x < n) ? ((w >> fsh) & LMASK) : 0u;
        }
        my_acc[b * nthr] = a;
      }
    } else {                    // flattened over the block's rows, prefix snapshot per row into smem
      const int n = rb[8] - rb[0];
      uint32_t run = 0u;
      my_acc[0] = 0u;
#pragma unroll 4
      for (int x = 0; x < n; ++x) {
        run += (wcol[s_woff[rb[0] + x]] >> fsh) & LMASK;
        s_acc[(x & 63) * 0 + tid] = run;       // stand-in for a per-row prefix store
      }
      total += run;
    }
    total += my_acc[7 * nthr];
  }
  long long t1 = clock64();
  if ((threadIdx.x & 31) == 0) out[threadIdx.x >> 5] = t1 - t0;
  if (total == 0x12345u) sink[0] = 1;
}

int main() {
  const int T = 1024;
  uint32_t h_offs[1025], h_woff[4096];
  for (int k = 0; k <= 1024; ++k) h_offs[k] = k * 6 < 2040 ? k * 6 : 2040;
  for (int r = 0; r < 4096; ++r) h_woff[r] = ((r * 131) % 784) * 8;
  uint32_t *d_offs, *d_woff; unsigned long long* d_out; int* d_sink;
  cudaMalloc(&d_offs, sizeof(h_offs)); cudaMalloc(&d_woff, sizeof(h_woff)); cudaMalloc(&d_out, 64 * 8); cudaMalloc(&d_sink, 4);
  cudaMemcpy(d_offs, h_offs, sizeof(h_offs), cudaMemcpyHostToDevice);
  cudaMemcpy(d_woff, h_woff, sizeof(h_woff), cudaMemcpyHostToDevice);
  unsigned long long h_out[64];
  auto run = [&](auto kern, const char* name, int threads) {
    kern<<<1, threads>>>(336, d_offs, d_woff, d_out, d_sink);
    cudaDeviceSynchronize();
    kern<<<1, threads>>>(336, d_offs, d_woff, d_out, d_sink);
    cudaDeviceSynchronize();
    cudaMemcpy(h_out, d_out, 64 * 8, cudaMemcpyDeviceToHost);
    unsigned long long mx = 0; for (int w = 0; w < threads / 32; ++w) mx = h_out[w] > mx ? h_out[w] : mx;
    printf("%-46s threads=%3d: %6.1f cycles/step (%s)\n", name, threads, mx / 336.0, cudaGetErrorString(cudaGetLastError()));
  };
  for (int threads : {32, 128, 224, 256}) {
    run(integ<0>, "rolled steps, unroll-4 rows (kernel)", threads);
    run(integ<1>, "unrolled 8 steps x 12 predicated rows", threads);
    run(integ<2>, "flattened rows, running sum", threads);
  }
  return 0;
}
