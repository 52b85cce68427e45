// Probe: per-step cost of the synchronisation primitives the SNN step loop can use on B200.
// (1) barrier.cluster arrive/wait with one DSMEM store per CTA per step, cluster sizes 1..16
// (2) hand-rolled grid barrier over global atomics, 148 CTAs
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("ERR %s at %d: %s\n",#x,__LINE__,cudaGetErrorString(e));}}while(0)

__device__ __forceinline__ uint32_t cluster_rank(){uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;":"=r"(r)); return r;}
__device__ __forceinline__ uint32_t cluster_n(){uint32_t r; asm volatile("mov.u32 %0, %%cluster_nctarank;":"=r"(r)); return r;}
__device__ __forceinline__ void st_remote_u64(void* p, uint32_t rank, unsigned long long v){
  uint32_t a = (uint32_t)__cvta_generic_to_shared(p); uint32_t ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;":"=r"(ra):"r"(a),"r"(rank));
  asm volatile("st.shared::cluster.u64 [%0], %1;"::"r"(ra),"l"(v):"memory");
}
__device__ __forceinline__ void cl_arrive(){asm volatile("barrier.cluster.arrive.release.aligned;":::"memory");}
__device__ __forceinline__ void cl_wait(){asm volatile("barrier.cluster.wait.acquire.aligned;":::"memory");}

__global__ void cluster_loop(int iters, unsigned long long* out, int dummy_smem){
  extern __shared__ unsigned long long sm[];
  unsigned long long* slots = sm; // [2][16]
  uint32_t r = cluster_rank(), n = cluster_n();
  unsigned long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    int par = it & 1;
    if (threadIdx.x < n) st_remote_u64(&slots[par*16 + r], threadIdx.x, (unsigned long long)(it*31+r));
    cl_arrive();
    cl_wait();
    if (threadIdx.x == 0) { unsigned long long m=0; for (uint32_t k=0;k<n;++k){unsigned long long x=slots[par*16+k]; m = x>m?x:m;} acc += m; }
    __syncthreads();
  }
  if (threadIdx.x == 0) out[blockIdx.x] = acc;
}

__global__ void grid_loop(int iters, unsigned* bar, unsigned long long* slots, unsigned long long* out){
  unsigned long long acc=0; unsigned nb = gridDim.x;
  for (int it = 0; it < iters; ++it) {
    __syncthreads();
    if (threadIdx.x == 0) {
      atomicMax(&slots[it & 1], (unsigned long long)(it*7 + blockIdx.x));
      __threadfence();
      unsigned target = (unsigned)(it+1) * nb;
      unsigned v = atomicAdd(bar, 1u) + 1u;
      while (v < target) { asm volatile("ld.acquire.gpu.u32 %0, [%1];":"=r"(v):"l"(bar)); }
      acc += *(volatile unsigned long long*)&slots[it & 1];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) out[blockIdx.x] = acc;
}

int main(){
  int dev=0; cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  printf("device %s SMs=%d smemPerBlockOptin=%zu clock=%d\n", p.name, p.multiProcessorCount, p.sharedMemPerBlockOptin, p.clockRate);
  unsigned long long* out; CK(cudaMalloc(&out, 4096*8));
  CK(cudaFuncSetAttribute(cluster_loop, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  int smem_sizes[3] = {1024, 100*1024, 200*1024};
  for (int si=0; si<3; ++si) {
    int smem = smem_sizes[si];
    CK(cudaFuncSetAttribute(cluster_loop, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    for (int cs = 1; cs <= 16; cs *= 2) {
      for (int threads : {128, 512}) {
        cudaLaunchConfig_t cfg = {}; cfg.gridDim = dim3(cs); cfg.blockDim = dim3(threads); cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = cs; at[0].val.clusterDim.y=1; at[0].val.clusterDim.z=1;
        cfg.attrs = at; cfg.numAttrs = 1;
        int ncl = -1; cudaError_t oe = cudaOccupancyMaxActiveClusters(&ncl, cluster_loop, &cfg);
        int iters = 20000;
        cudaError_t e = cudaLaunchKernelEx(&cfg, cluster_loop, 1000, out, 0); cudaDeviceSynchronize();
        cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
        cudaEventRecord(a); e = cudaLaunchKernelEx(&cfg, cluster_loop, iters, out, 0); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaError_t e2 = cudaGetLastError();
        float ms=0; cudaEventElapsedTime(&ms,a,b);
        printf("cluster cs=%2d threads=%3d smem=%6d maxActiveClusters=%d(%s) launch=%s: %.1f ns/step\n", cs, threads, smem, ncl, cudaGetErrorString(oe), cudaGetErrorString(e2!=cudaSuccess?e2:e), ms*1e6/iters);
      }
    }
  }
  unsigned* bar; unsigned long long* slots; CK(cudaMalloc(&bar, 4)); CK(cudaMalloc(&slots, 16));
  for (int nb : {16, 74, 148}) {
    for (int rep=0; rep<2; ++rep) {
      CK(cudaMemset(bar,0,4)); CK(cudaMemset(slots,0,16));
      int iters=5000; cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
      cudaEventRecord(a); grid_loop<<<nb,256>>>(iters,bar,slots,out); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms=0; cudaEventElapsedTime(&ms,a,b);
      printf("grid barrier ctas=%d: %.1f ns/step (%s)\n", nb, ms*1e6/iters, cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
