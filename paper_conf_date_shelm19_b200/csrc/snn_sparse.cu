// snn_sparse.cu -- NEXT-4: the Fig. 4 workload (§IV-A "an SNN of 10^3 LIF neurons and 10^4
// synapses", no learning; readings DESIGN.md R24-R26).  CUDA path only; shares nothing with oracle/.
//
// Design.  Trials (images x seeds) are independent: one CTA simulates one trial at a time
// and strides over the batch.  The synapse list is CSR by source (L1/L2-resident: 10^4 synapses = 37 KB);
// per step the CTA builds the list of active sources in shared memory (rate-coded input pixels drawn
// with the same Philox counters as the encoder, plus the neurons that spiked at t-1), scatters the codes
// of their synapses into per-neuron integer sums with shared-memory atomics (a warp per source, lanes
// over its synapses: integer adds, so the order does not matter), then runs the LIF recipe per neuron.
// Four barriers per step; membrane state, countdowns, sums and spike counts live in shared memory.
#include "snn_device.cuh"

namespace snn {

constexpr int kSparseThreads = 512;

template <bool FIXED>
__global__ void __launch_bounds__(kSparseThreads) sparse_kernel(const SparseDesc d) {
  extern __shared__ __align__(16) unsigned char smem[];
  const int n_lif = d.n_lif, n_in = d.n_in, T = d.T;
  unsigned long long* s_thr = reinterpret_cast<unsigned long long*>(smem);   // [256] encoder thresholds
  int* s_v = reinterpret_cast<int*>(smem + 256 * 8);        // [n_lif] fp32 bits or Q15.16
  int* s_cnt = s_v + n_lif;                                 // [n_lif] refractory countdown (R6)
  int* s_S = s_cnt + n_lif;                                 // [n_lif] eq.(3) integer sums
  int* s_src = s_S + n_lif;                                 // [n_in + n_lif] active sources of the step
  int* s_prev = s_src + n_in + n_lif;                       // [n_lif] neurons that spiked at t-1
  int* s_cnt_out = s_prev + n_lif;                          // [n_lif] spike counts of the trial
  int* s_n = s_cnt_out + n_lif;                             // [0] active sources, [1] spikes this step, [2] prev

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nw = blockDim.x >> 5;
  for (int x = tid; x < 256; x += blockDim.x) s_thr[x] = d.thr_enc[x];
  Lif lif;
  lif.af = d.af; lif.bf = d.bf; lif.cf = d.cf; lif.dtf = d.dtf; lif.kI = d.kI; lif.ief = d.ief; lif.vthf = d.vthf;
  lif.A = d.A; lif.B = d.B; lif.C = d.C; lif.E = d.E; lif.Vth = d.Vth; lif.fixed = FIXED;
  const int vinit = FIXED ? d.Vinit : __float_as_int(d.vinitf);
  const int vreset = FIXED ? d.Vreset : __float_as_int(d.vresetf);
  const int nq4 = (n_in + 3) >> 2;
  const int wl = (n_lif + 31) >> 5;
  unsigned long long act_sum = 0, spikes = 0;

  for (int tr = blockIdx.x; tr < d.n_trials; tr += gridDim.x) {
    const uint8_t* img = d.images + (size_t)tr * n_in;
    const unsigned long long seed = d.seeds[tr];
    uint32_t* cnt_out = d.counts + (size_t)tr * n_lif;
    for (int j = tid; j < n_lif; j += blockDim.x) { s_v[j] = vinit; s_cnt[j] = 0; s_S[j] = 0; s_cnt_out[j] = 0; }   // R5
    if (tid == 0) { s_n[0] = 0; s_n[1] = 0; s_n[2] = 0; }
    __syncthreads();
    for (int t = 0; t < T; ++t) {
      // ---- active sources: input pixels at t (encoder, R8 / R13) and the neurons that spiked at t-1 (R25)
      for (int g = tid; g < ((nq4 + 31) & ~31); g += blockDim.x) {
        uint32_t nib = 0;
        if (g < nq4) {
          const uint4 u = philox((uint32_t)t, (uint32_t)g, 0u, TAG_ENC, seed);
#pragma unroll
          for (int r = 0; r < 4; ++r) {
            const int i = 4 * g + r;
            if (i < n_in && (unsigned long long)pick(u, r) < s_thr[img[i]]) nib |= 1u << r;
          }
        }
        const int c = __popc(nib);
        int incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(FULL, incl, o);
          if (lane >= o) incl += y;
        }
        int base = 0;
        if (lane == 31 && incl) base = atomicAdd(&s_n[0], incl);
        base = __shfl_sync(FULL, base, 31);
        int pos = base + incl - c;
        while (nib) {
          const int r = __ffs(nib) - 1;
          nib &= nib - 1;
          s_src[pos++] = 4 * g + r;
        }
      }
      __syncthreads();
      const int n_act_in = s_n[0];
      const int n_prev = s_n[2];
      const int n_act = n_act_in + n_prev;
      // ---- eq.(3): scatter the codes of the active sources' synapses (8 lanes per source: ~10 synapses each)
      for (int a = warp * 4 + (lane >> 3); a < n_act; a += nw * 4) {
        const int s = a < n_act_in ? s_src[a] : n_in + s_prev[a - n_act_in];
        const int k0 = __ldg(&d.src_off[s]), k1 = __ldg(&d.src_off[s + 1]);
        for (int k = k0 + (lane & 7); k < k1; k += 8) atomicAdd(&s_S[__ldg(&d.tgt[k])], (int)__ldg(&d.q[k]));
      }
      if (tid == 0) act_sum += (unsigned long long)n_act_in;
      __syncthreads();
      // ---- eqs.(1)(2) + refractory (R6); no inhibition, no WTA (R26)
      for (int j = tid; j < n_lif; j += blockDim.x) {
        const int S = s_S[j];
        s_S[j] = 0;
        if (s_cnt[j] > 0) { --s_cnt[j]; continue; }
        int v = s_v[j];
        const bool x = lif.step_t<FIXED>(v, S);
        if (x) {
          v = vreset;
          s_cnt[j] = d.t_ref;
          const int p = atomicAdd(&s_n[1], 1);
          s_src[n_in + p] = j;                      // staging area of this step's spikes (after the inputs)
          ++s_cnt_out[j];
          ++spikes;
          if (d.raster) atomicOr(&d.raster[((size_t)tr * T + t) * wl + (j >> 5)], 1u << (j & 31));
        }
        s_v[j] = v;
      }
      __syncthreads();
      const int n_sp = s_n[1];
      for (int x = tid; x < n_sp; x += blockDim.x) s_prev[x] = s_src[n_in + x];
      __syncthreads();
      if (tid == 0) { s_n[2] = n_sp; s_n[1] = 0; s_n[0] = 0; }
      __syncthreads();
    }
    for (int j = tid; j < n_lif; j += blockDim.x) cnt_out[j] = (uint32_t)s_cnt_out[j];
  }
  if (d.stats) {
    if (tid == 0 && act_sum) atomicAdd(&d.stats[0], act_sum);
    if (spikes) atomicAdd(&d.stats[1], spikes);
  }
}

size_t sparse_smem_bytes(int n_in, int n_lif) {
  return (size_t)(3 * n_lif + n_in + n_lif + n_lif + n_lif + 4) * 4 + 256 * 8;
}

template <bool FIXED>
static cudaError_t launch_sparse_t(const SparseDesc& d, int grid, int nthr, size_t smem, cudaStream_t s) {
  auto k = sparse_kernel<FIXED>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k<<<grid, nthr, smem, s>>>(d);
  return cudaGetLastError();
}

cudaError_t sparse_occupancy(int fixed, int nthr, size_t smem, int* out) {
  cudaError_t e;
  if (fixed) {
    e = cudaFuncSetAttribute(sparse_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(out, sparse_kernel<true>, nthr, smem);
  }
  e = cudaFuncSetAttribute(sparse_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(out, sparse_kernel<false>, nthr, smem);
}

cudaError_t launch_sparse(const SparseDesc& d, int grid, int nthr, size_t smem, int fixed, cudaStream_t s) {
  if (d.n_trials <= 0 || d.T <= 0) return cudaSuccess;
  return fixed ? launch_sparse_t<true>(d, grid, nthr, smem, s) : launch_sparse_t<false>(d, grid, nthr, smem, s);
}

}  // namespace snn
