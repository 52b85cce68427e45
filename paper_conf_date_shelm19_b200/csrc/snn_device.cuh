// snn_device.cuh -- device helpers shared by the CUDA kernels (CUDA path only).
#pragma once
#include <cstdint>
#include "snn_internal.h"

namespace snn {

constexpr unsigned FULL = 0xFFFFFFFFu;

// Philox4x32-10 (Salmon et al. SC'11), counter (c0,c1,c2,c3), key (seed lo, seed hi)  [R13]
__device__ __forceinline__ uint4 philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                        unsigned long long seed) {
  uint32_t k0 = (uint32_t)seed, k1 = (uint32_t)(seed >> 32);
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
    const uint32_t lo0 = 0xD2511F53u * c0, hi0 = __umulhi(0xD2511F53u, c0);
    const uint32_t lo1 = 0xCD9E8D57u * c2, hi1 = __umulhi(0xCD9E8D57u, c2);
    const uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0; c1 = lo1; c2 = n2; c3 = lo0;
  }
  return make_uint4(c0, c1, c2, c3);
}

__device__ __forceinline__ uint32_t pick(const uint4& u, int l) {
  return l == 0 ? u.x : (l == 1 ? u.y : (l == 2 ? u.z : u.w));
}

// ---- cluster primitives (sm_90+; barrier.cluster is a hardware cluster-wide barrier)
__device__ __forceinline__ void cluster_arrive() {
  asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_arrive_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() {
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t map_cluster(const void* local, uint32_t rank) {
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(local);
  uint32_t ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank));
  return ra;
}
// store into the same shared variable of CTA `rank` (DSMEM)
__device__ __forceinline__ void st_cluster_u64(unsigned long long* local, uint32_t rank, unsigned long long v) {
  asm volatile("st.shared::cluster.u64 [%0], %1;" ::"r"(map_cluster(local, rank)), "l"(v) : "memory");
}
// fire-and-forget min into the same shared int of CTA `rank`
__device__ __forceinline__ void red_min_cluster(int* local, uint32_t rank, int v) {
  asm volatile("red.relaxed.cluster.shared::cluster.min.s32 [%0], %1;" ::"r"(map_cluster(local, rank)), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ int ld_volatile_shared_u32addr(uint32_t a) {
  int v;
  asm volatile("ld.volatile.shared.s32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int ld_volatile_shared(const int* p) {
  int v;
  asm volatile("ld.volatile.shared.s32 %0, [%1];" : "=r"(v) : "r"((uint32_t)__cvta_generic_to_shared(p)));
  return v;
}

__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// ---- system-scope mailbox primitives (cross-GPU shard exchange over NVLink peer memory)
__device__ __forceinline__ void st_relaxed_sys_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed_sys_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_relaxed_sys_s32(const int* p) {
  int v;
  asm volatile("ld.relaxed.sys.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_max_sys_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("red.relaxed.sys.global.max.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// order-preserving map of an fp32 bit pattern to u32 (WTA argmax key)
__device__ __forceinline__ uint32_t float_ord(uint32_t u) {
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}

// ---- LIF recipes; v is the fp32 bit pattern or Q15.16
struct Lif {
  float af, bf, cf, dtf, kI, ief, vthf;
  long long A, B, C, E;
  int Vth;
  bool fixed;
  __device__ __forceinline__ void load(const NetDesc& d) {
    af = d.af; bf = d.bf; cf = d.cf; dtf = d.dtf; kI = d.kI; ief = d.ief; vthf = d.vthf;
    A = d.A; B = d.B; C = d.C; E = d.E; Vth = d.Vth; fixed = d.membrane_mode == 1;
  }
  // one Euler step of a non-refractory neuron; returns true iff v crosses the threshold (eq.(2) "v > v_th")
  __device__ __forceinline__ bool step(int& v, int S) const {
    if (fixed) {
      const long long x = v;
      const long long bv = (B * x + (1LL << 31)) >> 32;
      const long long cterm = (C * (long long)S + (1LL << 15)) >> 16;
      v = (int)(x + A + bv + cterm + E);
      return v > Vth;
    }
    const float vf = __int_as_float(v);
    const float I = __fmul_rn(__int2float_rn(S), kI);
    const float xx = __fadd_rn(I, ief);
    const float y = __fmaf_rn(cf, xx, af);
    const float dv = __fmaf_rn(bf, vf, y);
    const float vn = __fmaf_rn(dtf, dv, vf);
    v = __float_as_int(vn);
    return vn > vthf;
  }
  template <bool FIXED>
  __device__ __forceinline__ bool step_t(int& v, int S) const {
    if constexpr (FIXED) {
      const long long x = v;
      const long long bv = (B * x + (1LL << 31)) >> 32;
      const long long cterm = (C * (long long)S + (1LL << 15)) >> 16;
      v = (int)(x + A + bv + cterm + E);
      return v > Vth;
    } else {
      const float vf = __int_as_float(v);
      const float I = __fmul_rn(__int2float_rn(S), kI);
      const float xx = __fadd_rn(I, ief);
      const float y = __fmaf_rn(cf, xx, af);
      const float dv = __fmaf_rn(bf, vf, y);
      const float vn = __fmaf_rn(dtf, dv, vf);
      v = __float_as_int(vn);
      return vn > vthf;
    }
  }
  // step_t split in two: the part of eq.(1) that does not depend on v (computable ahead for a block of steps)
  // and the v-dependent rest; post_t(v, pre_t(S)) performs exactly the operations of step_t(v, S) (the integer
  // recipe's int64 sum is reassociated, which is exact)
  template <bool FIXED>
  __device__ __forceinline__ int pre_t(int S) const {
    if constexpr (FIXED) {
      return (int)(A + ((C * (long long)S + (1LL << 15)) >> 16) + E);
    } else {
      const float I = __fmul_rn(__int2float_rn(S), kI);
      return __float_as_int(__fmaf_rn(cf, __fadd_rn(I, ief), af));
    }
  }
  template <bool FIXED>
  __device__ __forceinline__ bool post_t(int& v, int y) const {
    if constexpr (FIXED) {
      const long long x = v;
      v = (int)(x + (long long)y + ((B * x + (1LL << 31)) >> 32));
      return v > Vth;
    } else {
      const float vf = __int_as_float(v);
      const float dv = __fmaf_rn(bf, vf, __int_as_float(y));
      const float vn = __fmaf_rn(dtf, dv, vf);
      v = __float_as_int(vn);
      return vn > vthf;
    }
  }
  __device__ __forceinline__ uint32_t ord(int v) const {
    return fixed ? ((uint32_t)v ^ 0x80000000u) : float_ord((uint32_t)v);
  }
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

}  // namespace snn
