// Probe 2: per-step cost of a polled DSMEM all-to-all exchange of a tagged u64 key
// (each CTA: CTA-local reduce -> lanes 0..CS-1 store key to slot[par][rank] of every CTA ->
// every warp polls its local slots until the tag matches -> warp redux).  Compare with syncthreads only.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t cluster_rank(){uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;":"=r"(r)); return r;}
__device__ __forceinline__ uint32_t cluster_n(){uint32_t r; asm volatile("mov.u32 %0, %%cluster_nctarank;":"=r"(r)); return r;}
__device__ __forceinline__ void st_remote_u64(const void* p, uint32_t rank, unsigned long long v){
  uint32_t a = (uint32_t)__cvta_generic_to_shared(p); uint32_t ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;":"=r"(ra):"r"(a),"r"(rank));
  asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;"::"r"(ra),"l"(v):"memory");
}
__device__ __forceinline__ unsigned long long ld_local_u64(const void* p){
  uint32_t a = (uint32_t)__cvta_generic_to_shared(p); unsigned long long v;
  asm volatile("ld.relaxed.cluster.shared::cta.u64 %0, [%1];":"=l"(v):"r"(a):"memory"); return v;
}
__global__ void xchg_loop(int iters, unsigned long long* out, int mode){
  __shared__ unsigned long long slots[2][16];
  __shared__ unsigned long long wkeys[32];
  uint32_t r = cluster_rank(), n = cluster_n();
  int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (threadIdx.x < 32) { slots[0][threadIdx.x & 15] = 0; slots[1][threadIdx.x & 15] = 0; }
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;":::"memory");
  unsigned long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    unsigned long long mykey = ((unsigned long long)((it * 2654435761u) ^ threadIdx.x ^ (r << 20)) << 12);
    // warp reduce (two-pass 32-bit redux)
    unsigned hi = (unsigned)(mykey >> 32), lo = (unsigned)mykey;
    unsigned mh = __reduce_max_sync(0xffffffffu, hi);
    unsigned ml = __reduce_max_sync(0xffffffffu, hi == mh ? lo : 0u);
    if (lane == 0) wkeys[warp] = ((unsigned long long)mh << 32) | ml;
    __syncthreads();
    if (mode == 0) { // syncthreads only: CTA reduce
      if (warp == 0) { unsigned long long k = lane < nw ? wkeys[lane] : 0; hi=(unsigned)(k>>32); lo=(unsigned)k;
        mh = __reduce_max_sync(0xffffffffu, hi); ml = __reduce_max_sync(0xffffffffu, hi==mh?lo:0u); if (lane==0) wkeys[31] = ((unsigned long long)mh<<32)|ml; }
      __syncthreads();
      acc += wkeys[31];
    } else {
      unsigned tag = (it >> 1) & 1u, par = it & 1;
      if (warp == 0) {
        unsigned long long k = lane < nw ? wkeys[lane] : 0; hi=(unsigned)(k>>32); lo=(unsigned)k;
        mh = __reduce_max_sync(0xffffffffu, hi); ml = __reduce_max_sync(0xffffffffu, hi==mh?lo:0u);
        unsigned long long ck = (((unsigned long long)mh<<32)|ml) & ~1ull; ck |= tag;
        if (lane < n) st_remote_u64(&slots[par][r], lane, ck);
      }
      // every warp polls
      unsigned long long v = 0;
      if (lane < n) { do { v = ld_local_u64(&slots[par][lane]); } while ((unsigned)(v & 1ull) != tag); }
      hi=(unsigned)(v>>32); lo=(unsigned)v & ~1u;
      mh = __reduce_max_sync(0xffffffffu, hi); ml = __reduce_max_sync(0xffffffffu, hi==mh?lo:0u);
      acc += ((unsigned long long)mh<<32)|ml;
      __syncwarp();
      // slot reuse safety comes from the 2-deep ring + the tag; wkeys reuse needs a barrier:
      __syncthreads();
    }
  }
  if (threadIdx.x == 0) out[blockIdx.x] = acc;
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;":::"memory");
}
int main(){
  unsigned long long* out; cudaMalloc(&out, 4096*8);
  cudaFuncSetAttribute(xchg_loop, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int mode = 0; mode < 2; ++mode)
  for (int cs = 1; cs <= 16; cs *= 2) for (int threads : {128, 416}) {
    cudaLaunchConfig_t cfg = {}; cfg.gridDim = dim3(cs); cfg.blockDim = dim3(threads); cfg.dynamicSmemBytes = 0;
    cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = cs; at[0].val.clusterDim.y=1; at[0].val.clusterDim.z=1;
    cfg.attrs = at; cfg.numAttrs = 1;
    int iters = 20000;
    cudaLaunchKernelEx(&cfg, xchg_loop, 1000, out, mode); cudaDeviceSynchronize();
    cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a); cudaLaunchKernelEx(&cfg, xchg_loop, iters, out, mode); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms=0; cudaEventElapsedTime(&ms,a,b);
    printf("mode=%s cs=%2d threads=%3d: %.1f ns/step (%s)\n", mode? "dsmem-poll":"syncthreads", cs, threads, ms*1e6/iters, cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
