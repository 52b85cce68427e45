// snn_infer.cu -- NEXT-1: batch-parallel inference with frozen weights, neuron labelling and the class
// vote (§III-B "After learning is complete, the first 1000 images in the test set are used to
// label all the neurons in the first layer. The rest of the test set ... are used for inference";
// readings DESIGN.md R21-R23).  CUDA path only; shares nothing with oracle/.
//
// Design.  Images are independent once the weights are frozen, so one CTA simulates
// one image at a time (persistent grid, images strided over CTAs) with no cross-SM synchronisation:
//   * consumer threads own 32 consecutive columns each: v in registers, the refractory / inhibition
//     countdown as an absolute "free from step" (u16, packed two per register);
//   * a producer warp streams the weight rows of the active inputs of upcoming steps from global
//     memory (L2-resident, inference layout: codes bit-packed row-major) into a shared-memory ring
//     with cp.async.bulk (TMA bulk copies), one mbarrier per ring slot, running up to kSR steps ahead
//     of the consumers (also across image boundaries);
//   * integration (eq.(3)) is SWAR: one shift+mask+add per (word, lane group) adds 4 (2-bit) or 2
//     (4/8-bit) columns at once into byte / half-word lanes;
//   * the LIF update (eqs.(1)(2), DESIGN.md §3.3 recipes) runs only for non-held columns; a thread whose
//     columns are all held skips the step;
//   * one barrier per step (bar.red.or of "some column crossed"); only then a CTA-wide u64 argmax
//     (HARD) or spiker count (LAYER) and the WTA / inhibition update (R7).
// Steps whose active-row count exceeds the ring budget fall back to per-column direct loads (rare:
// saturating inputs).
#include "snn_device.cuh"

namespace snn {

constexpr int kSR = 64;                  // step ring of the producer's per-step (base, count) records
constexpr uint32_t kDirect = 0x80000000u;
constexpr int kWB = 8;                   // steps per producer word-prefetch batch (cp.async, double-buffered)
constexpr int kInfMaxThreads = 256;      // <= 224 column threads (n_exc <= 7168) + the producer warp: 255 registers

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  while (!mbar_test(bar, parity)) {
  }
}
__device__ __forceinline__ uint32_t ld_acquire_cta(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.cta.shared.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_cta(uint32_t* p, uint32_t v) {
  asm volatile("st.release.cta.shared.u32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}
// named barriers among the consumer warps (the producer warp never joins them)
__device__ __forceinline__ int bar_red_or(int id, int n, bool pred) {
  int r;
  asm volatile("{\n .reg .pred p, q;\n setp.ne.u32 q, %1, 0;\n bar.red.or.pred p, %2, %3, q;\n selp.s32 %0, 1, 0, p;\n}\n"
               : "=r"(r) : "r"((uint32_t)pred), "r"(id), "r"(n) : "memory");
  return r;
}
__device__ __forceinline__ void bar_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
// TMA bulk copy global -> shared, completion signalled on `bar` (bytes % 16 == 0, 16-byte aligned)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

// SWAR geometry of one thread's 32 columns at BITS bits per code:
//   word k (of BITS words) holds columns k*FPW .. k*FPW+FPW-1 (field f at bits f*BITS);
//   lane width LW (8 for 2-bit, 16 otherwise); acc[k][m] lane l accumulates field f = l*M + m.
template <int BITS>
struct Swar {
  static constexpr int FPW = 32 / BITS;
  static constexpr int LW = BITS == 2 ? 8 : 16;
  static constexpr int LPW = 32 / LW;
  static constexpr int M = FPW / LPW;
  static constexpr int NACC = BITS * M;
  static constexpr uint32_t MASK = BITS == 2 ? 0x03030303u : (BITS == 4 ? 0x000F000Fu : 0x00FF00FFu);
  __device__ static __forceinline__ void add(uint32_t (&acc)[NACC], const uint32_t (&w)[BITS]) {
#pragma unroll
    for (int k = 0; k < BITS; ++k)
#pragma unroll
      for (int m = 0; m < M; ++m) acc[k * M + m] += (w[k] >> (m * BITS)) & MASK;
  }
  __device__ static __forceinline__ int get(const uint32_t (&acc)[NACC], int c) {
    const int k = c / FPW, f = c % FPW, l = f / M, m = f % M;
    return (int)((acc[k * M + m] >> (l * LW)) & ((1u << LW) - 1u));
  }
};

template <int BITS, bool FIXED, int MINB>
__global__ void __launch_bounds__(kInfMaxThreads, MINB) infer_kernel(const InferDesc d) {
  using SW = Swar<BITS>;
  extern __shared__ __align__(128) unsigned char smem[];
  unsigned char* ring = smem;                                                   // [R][row_bytes]
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)d.R * d.row_bytes);  // [R]
  uint32_t* s_nrows = reinterpret_cast<uint32_t*>(full + d.R);                  // [kSR] rows (| kDirect)
  uint32_t* s_base = s_nrows + kSR;                                             // [kSR] first ring position
  unsigned long long* s_key = reinterpret_cast<unsigned long long*>(s_base + kSR);  // [32]
  int* s_cnt = reinterpret_cast<int*>(s_key + 32);                              // [32]
  uint32_t* s_wbuf = reinterpret_cast<uint32_t*>(s_cnt + 32);                   // [2][kWB][32] producer's word prefetch
  uint32_t* s_pub = s_wbuf + 2 * kWB * 32;   // steps whose ring records the producer has published
  uint32_t* s_rel = s_pub + 1;               // steps the consumers have finished (their ring slots are free)

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int ncw = (d.nthr_cols + 31) >> 5;        // consumer warps
  const bool is_producer = warp == ncw;
  const int T = d.T;
  const uint32_t Ru = (uint32_t)d.R;               // ring slots (any R in [8, 64]); positions are u32 per CTA
  const int my_images = d.n_images > (int)blockIdx.x ? (d.n_images - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
  const long long G = (long long)my_images * T;   // steps this CTA simulates (images back to back)
  if (G == 0) return;

  if (tid == 0) {
    for (int r = 0; r < d.R; ++r) mbar_init(&full[r], 1);
    *s_pub = 0u;
    *s_rel = 0u;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int ncons = ncw * 32;                     // consumer threads: they alone take part in the step barriers

  // ---------------- producer state (producer warp, uniform across its lanes)
  long long p_step = 0;       // next step to issue
  int p_img = 0, p_t = 0;     // its image (of this CTA) and timestep
  long long p_pos = 0;        // next ring position (consumers see its low 32 bits; R | 2^32)
  unsigned long long p_act = 0;   // active input rows of the issued steps
  // Issue steps [p_step, min(G, limit)) while their rows fit the ring; ring positions before the first
  // row of step `first_live` are released (their readers passed a barrier).  Steps with more than rmax
  // rows are marked direct (read from global memory by the consumers, no ring slots).
  // Encoded input words of upcoming steps (n_in <= 1024: one word per lane) are prefetched by the producer
  // warp with cp.async in batches of kWB steps, two batches in flight, so that issuing a step never waits
  // on a global-memory round trip.
  const bool wfast = d.nwi <= 32;
  long long pf_step = 0;      // next step to prefetch
  long long wb_entered = -1;  // last batch whose words the producer started to read
  int pf_img = 0, pf_t = 0;
  auto prefetch_batch = [&]() {
    uint32_t* dst = s_wbuf + ((pf_step / kWB) & 1) * (kWB * 32);
#pragma unroll 1
    for (int q = 0; q < kWB; ++q) {
      if (pf_step < G && lane < d.nwi) {
        const long long k = (long long)blockIdx.x + (long long)pf_img * gridDim.x;
        const uint32_t* src = d.words + ((size_t)k * T + pf_t) * d.nwi + lane;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst + q * 32 + lane)), "l"(src) : "memory");
      }
      ++pf_step;
      if (++pf_t == T) { pf_t = 0; ++pf_img; }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  auto produce = [&](long long limit, long long first_live) {
    long long released = p_pos;
    if (first_live < p_step) released = p_pos - (long long)(uint32_t)((uint32_t)p_pos - s_base[first_live & (kSR - 1)]);
    const uint32_t row_bytes = (uint32_t)d.row_bytes;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // consumers' generic reads before TMA rewrites
    while (p_step < limit && p_step < G) {
      const int s = (int)(p_step & (kSR - 1));
      const long long k = (long long)blockIdx.x + (long long)p_img * gridDim.x;
      const uint32_t* wr = d.words + ((size_t)k * T + p_t) * d.nwi;
      uint32_t w_l = 0;                                // this lane's word of the step (fast path)
      int n = 0;
      if (wfast) {
        if (p_step / kWB > wb_entered) {   // entering batch b: refill the buffer of batch b-1 with batch b+1,
          wb_entered = p_step / kWB;       // then wait for batch b (each lane reads only its own words)
          if (p_step > 0) prefetch_batch();
          asm volatile("cp.async.wait_group 1;" ::: "memory");
        }
        w_l = lane < d.nwi ? s_wbuf[((p_step / kWB) & 1) * (kWB * 32) + (p_step % kWB) * 32 + lane] : 0u;
        n = __popc(w_l);
      } else {
        for (int w = lane; w < d.nwi; w += 32) n += __popc(__ldg(&wr[w]));
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) n += __shfl_xor_sync(FULL, n, o);
      if (n <= d.rmax && (long long)d.R - (p_pos - released) < n) break;   // ring full: after the next barrier
      if (n > d.rmax) {
        if (lane == 0) { s_base[s] = (uint32_t)p_pos; s_nrows[s] = (uint32_t)n | kDirect; }
      } else {
        long long pos = p_pos;
        for (int w0 = 0; w0 < d.nwi; w0 += 32) {
          const int w = w0 + lane;
          uint32_t bits = wfast ? w_l : (w < d.nwi ? __ldg(&wr[w]) : 0u);
          const int c = __popc(bits);
          int incl = c;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
          }
          long long p = pos + (incl - c);
          while (bits) {                               // rows in ascending order, one bulk copy each
            const int i = 32 * w + __ffs(bits) - 1;
            bits &= bits - 1;
            const uint32_t pu = (uint32_t)p, use = pu / Ru, slot = pu - use * Ru;
            if (p >= d.R) mbar_wait(&full[slot], (use - 1u) & 1u);                  // previous use landed
            mbar_arrive_tx(&full[slot], row_bytes);
            bulk_g2s(ring + (size_t)slot * row_bytes, d.w + (size_t)i * d.wpr, row_bytes, &full[slot]);
            ++p;
          }
          pos += __shfl_sync(FULL, incl, 31);
        }
        if (lane == 0) { s_base[s] = (uint32_t)p_pos; s_nrows[s] = (uint32_t)n; }
        p_pos = pos;
      }
      p_act += (unsigned long long)n;                 // active rows of the step (stats [0])
      ++p_step;
      if (++p_t == T) { p_t = 0; ++p_img; }
    }
  };

  // ---------------- consumer state: 32 columns per thread
  const int tcol = tid;                          // column-thread index (consumers only)
  const int j0 = 32 * tcol;
  int v[32];
  uint32_t fr[16];                               // free-from step, u16 x 2 (column c at half c & 1 of fr[c >> 1])
  int my_min_free = 0;                           // min / max over this thread's columns (padding: 0xFFFF)
  int my_max_free = 0;
  const int vinit = FIXED ? d.Vinit : __float_as_int(d.vinitf);
  const int vreset = FIXED ? d.Vreset : __float_as_int(d.vresetf);
  Lif lif;
  lif.af = d.af; lif.bf = d.bf; lif.cf = d.cf; lif.dtf = d.dtf; lif.kI = d.kI; lif.ief = d.ief; lif.vthf = d.vthf;
  lif.A = d.A; lif.B = d.B; lif.C = d.C; lif.E = d.E; lif.Vth = d.Vth; lif.fixed = FIXED;
  const bool consumer = !is_producer && tcol < d.nthr_cols;
  unsigned long long spikes = 0, lif_cs = 0;   // lif_cs: column-steps that ran eqs.(1)(2)

  if (is_producer) {
    // the producer runs decoupled from the consumers' step barriers: it publishes step records (release) and
    // reuses ring slots of steps the consumers report finished (acquire)
    if (wfast) { prefetch_batch(); prefetch_batch(); }
    uint32_t rel = 0;
    while (p_step < G) {
      const long long before = p_step;
      produce((long long)rel + kSR - 1, (long long)rel);
      if (p_step != before) {
        __syncwarp();
        if (lane == 0) st_release_cta(s_pub, (uint32_t)p_step);
      }
      uint32_t r2 = ld_acquire_cta(s_rel);
      while (r2 == rel && p_step == before && p_step < G) r2 = ld_acquire_cta(s_rel);   // ring full: wait
      rel = __shfl_sync(FULL, r2, 0);
    }
    if (d.stats && lane == 0 && p_act) atomicAdd(&d.stats[0], p_act);
    return;
  }

  uint32_t* counts_img = nullptr;
  int img = 0, t = 0;
  for (long long g = 0; g < G; ++g, (++t == T ? (t = 0, ++img) : 0)) {
    const uint32_t tt = (uint32_t)t;
    bool has_cand = false;
    unsigned long long best = 0;
    int ncand = 0;
    if (t == 0) {
      const long long k = (long long)blockIdx.x + (long long)img * gridDim.x;
      counts_img = d.counts + (size_t)k * d.n_exc;
      if (consumer) {
        my_min_free = 0;
#pragma unroll
        for (int c = 0; c < 32; ++c) v[c] = vinit;
#pragma unroll
        for (int h = 0; h < 16; ++h) {
          const uint32_t lo = (j0 + 2 * h < d.n_exc) ? 0u : 0xFFFFu;      // padding columns never integrate
          const uint32_t hi = (j0 + 2 * h + 1 < d.n_exc) ? 0u : 0xFFFFu;
          fr[h] = lo | (hi << 16);
        }
        my_max_free = j0 + 32 > d.n_exc ? 0xFFFF : 0;
        if (j0 + 32 > d.n_exc) my_min_free = j0 >= d.n_exc ? 0xFFFF : 0;
      }
    }
    // a thread whose 32 columns are all held (R6, R7) reads no rows: it goes straight to the step's barrier
    if (consumer && (int)tt >= my_min_free) {
      while (ld_acquire_cta(s_pub) <= (uint32_t)g) {}     // the producer published step g
      const uint32_t nr = s_nrows[g & (kSR - 1)];
      if (!(nr & kDirect)) {
        uint32_t acc[SW::NACC];
#pragma unroll
        for (int a = 0; a < SW::NACC; ++a) acc[a] = 0;
        const uint32_t pos0 = s_base[g & (kSR - 1)];
        uint32_t par = pos0 / Ru;
        uint32_t slot = pos0 - par * Ru;
        par &= 1u;
        for (uint32_t r = 0; r < nr; ++r) {
          mbar_wait(&full[slot], par);
          const uint32_t* src = reinterpret_cast<const uint32_t*>(ring + (size_t)slot * d.row_bytes) + tcol * BITS;
          uint32_t w[BITS];
          if constexpr (BITS == 2) {
            const uint2 x = *reinterpret_cast<const uint2*>(src);
            w[0] = x.x; w[1] = x.y;
          } else {
#pragma unroll
            for (int q = 0; q < BITS / 4; ++q) {
              const uint4 x = reinterpret_cast<const uint4*>(src)[q];
              w[4 * q] = x.x; w[4 * q + 1] = x.y; w[4 * q + 2] = x.z; w[4 * q + 3] = x.w;
            }
          }
          SW::add(acc, w);
          if (++slot == Ru) { slot = 0; par ^= 1u; }
        }
        // LIF (eqs.(1)(2)) of the non-held columns; keys only if some column crossed
        bool cross = false;
        if ((int)tt >= my_max_free) {                             // no column of this thread is held
#pragma unroll
          for (int c = 0; c < 32; ++c) cross |= lif.step_t<FIXED>(v[c], SW::get(acc, c));
          lif_cs += 32;
        } else {
#pragma unroll
          for (int c = 0; c < 32; ++c) {
            const uint32_t f = (fr[c >> 1] >> ((c & 1) * 16)) & 0xFFFFu;
            if (tt >= f) { cross |= lif.step_t<FIXED>(v[c], SW::get(acc, c)); ++lif_cs; }   // held: keep v (R6, R7)
          }
        }
        if (cross) {
#pragma unroll
          for (int c = 0; c < 32; ++c) {
            const uint32_t f = (fr[c >> 1] >> ((c & 1) * 16)) & 0xFFFFu;
            const bool above = FIXED ? (v[c] > d.Vth) : (__int_as_float(v[c]) > d.vthf);
            if (tt >= f && above) {
              const unsigned long long key = ((unsigned long long)lif.ord(v[c]) << 32) | (0xFFFFFFFFu - (uint32_t)(j0 + c));
              best = key > best ? key : best;
              ++ncand;
            }
          }
        }
      } else {
        // direct: more active rows than the ring budget -- per column, codes straight from global memory
        const int k_img = blockIdx.x + img * gridDim.x;
        const uint32_t* wr = d.words + ((size_t)k_img * T + t) * d.nwi;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const uint32_t f = (fr[c >> 1] >> ((c & 1) * 16)) & 0xFFFFu;
          if (tt < f) continue;
          const int kw = c / SW::FPW, sh = (c % SW::FPW) * BITS;
          int S = 0;
          for (int w = 0; w < d.nwi; ++w) {
            uint32_t bits = __ldg(&wr[w]);
            while (bits) {
              const int i = 32 * w + __ffs(bits) - 1;
              bits &= bits - 1;
              S += (int)((__ldg(&d.w[(size_t)i * d.wpr + tcol * BITS + kw]) >> sh) & ((1u << BITS) - 1u));
            }
          }
          ++lif_cs;
          if (lif.step_t<FIXED>(v[c], S)) {
            const unsigned long long key = ((unsigned long long)lif.ord(v[c]) << 32) | (0xFFFFFFFFu - (uint32_t)(j0 + c));
            best = key > best ? key : best;
            ++ncand;
          }
        }
      }
      has_cand = ncand > 0;
    }
    // ---- B_g: the one barrier of a step (consumers only); then the ring slots of step g are released
    const int any = bar_red_or(1, ncons, has_cand);
    if (tid == 0) st_release_cta(s_rel, (uint32_t)(g + 1));
    if (any) {
      // WTA (R7): HARD -> the largest key wins; LAYER -> every candidate spikes
      unsigned long long wb = best;
      int wc = ncand;
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        const unsigned long long y = __shfl_xor_sync(FULL, wb, o);
        wb = y > wb ? y : wb;
        wc += __shfl_xor_sync(FULL, wc, o);
      }
      if (lane == 0) { s_key[warp] = wb; s_cnt[warp] = wc; }
      bar_sync(2, ncons);
      unsigned long long kbest = 0;
      int nsp = 0;
      for (int q = 0; q < ncw; ++q) {
        const unsigned long long y = s_key[q];
        kbest = y > kbest ? y : kbest;
        nsp += s_cnt[q];
      }
      bar_sync(2, ncons);                                // s_key / s_cnt reusable
      const int W = (int)(0xFFFFFFFFu - (uint32_t)kbest);
      if (d.wta_mode == 0) nsp = 1;
      if (consumer) {
        const uint32_t f_ref = min(tt + 1u + (uint32_t)d.t_ref, 0xFFFFu);
        const uint32_t f_inh = min(tt + 1u + (uint32_t)d.t_inh, 0xFFFFu);
        int mn = 0xFFFF, mx = 0;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const int j = j0 + c;
          const int sh = (c & 1) * 16;
          uint32_t f = (fr[c >> 1] >> sh) & 0xFFFFu;
          if (j < d.n_exc) {
            bool spk;
            if (d.wta_mode == 0) {
              spk = j == W;
            } else {   // LAYER: this column spikes iff it crossed at this step (held columns did not integrate)
              spk = ((int)tt >= (int)f) &&
                    (FIXED ? (v[c] > d.Vth) : (__int_as_float(v[c]) > d.vthf));
            }
            if (spk) {
              v[c] = vreset;                               // eq.(2)
              f = f_ref;
              counts_img[j] += 1u;
              ++spikes;
            }
            if (nsp >= 2 || !spk) {                        // "all other neurons ... for t_inh"
              f = max(f, f_inh);
              if (d.inh_mode == 0) v[c] = vreset;
            }
            fr[c >> 1] = (fr[c >> 1] & ~(0xFFFFu << sh)) | (f << sh);
          }
          mn = min(mn, (int)f);
          mx = max(mx, (int)f);
        }
        my_min_free = mn;
        my_max_free = mx;
      }
    }
  }
  if (d.stats && consumer && spikes) atomicAdd(&d.stats[1], spikes);
  if (d.stats && consumer && lif_cs) atomicAdd(&d.stats[2], lif_cs);
}

// Pack u8 codes [n_in][n_exc] into the inference layout: row i, word q = column-thread q / BITS ...
// column j at word (j / FPW) bits (j % FPW) * BITS; rows padded to wpr words with zeros.
__global__ void pack_infer_kernel(const uint8_t* __restrict__ codes, int n_in, int n_exc, int bits, int wpr,
                                  uint32_t* __restrict__ w) {
  const size_t gid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= (size_t)n_in * wpr) return;
  const int i = (int)(gid / wpr), q = (int)(gid % wpr);
  const int fpw = 32 / bits;
  uint32_t word = 0;
  for (int f = 0; f < fpw; ++f) {
    const int j = q * fpw + f;
    if (j < n_exc) word |= (uint32_t)codes[(size_t)i * n_exc + j] << (f * bits);
  }
  w[gid] = word;
}

// R22: labels[j] = argmax_c (sum_{k in c} counts[k][j]) / N_c, ties -> lowest c, -1 if silent.
// One thread per neuron; exact comparison of the ratios as 128-bit cross products.
__device__ __forceinline__ bool ratio_gt(unsigned long long ra, unsigned long long na, unsigned long long rb,
                                         unsigned long long nb) {
  const unsigned long long h1 = __umul64hi(ra, nb), l1 = ra * nb;
  const unsigned long long h2 = __umul64hi(rb, na), l2 = rb * na;
  return h1 > h2 || (h1 == h2 && l1 > l2);
}

__global__ void label_kernel(const uint32_t* __restrict__ counts, int n_images, int n_exc,
                             const int32_t* __restrict__ classes, int n_classes, int32_t* __restrict__ labels) {
  __shared__ unsigned long long s_N[kMaxClasses];
  for (int c = threadIdx.x; c < n_classes; c += blockDim.x) s_N[c] = 0;
  __syncthreads();
  for (int k = threadIdx.x; k < n_images; k += blockDim.x) atomicAdd(&s_N[classes[k]], 1ull);
  __syncthreads();
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n_exc) return;
  unsigned long long r[kMaxClasses];
  for (int c = 0; c < n_classes; ++c) r[c] = 0;
  for (int k = 0; k < n_images; ++k) r[__ldg(&classes[k])] += __ldg(&counts[(size_t)k * n_exc + j]);
  int best = -1;
  for (int c = 0; c < n_classes; ++c) {
    if (s_N[c] == 0 || r[c] == 0) continue;
    if (best < 0 || ratio_gt(r[c], s_N[c], r[best], s_N[best])) best = c;
  }
  labels[j] = best;
}

// R23: pred[k] = argmax_c (sum_{j: label_j = c} counts[k][j]) / M_c, ties -> lowest c, -1 if no vote.
// One warp per image.
constexpr int kVoteWarps = 8;
__global__ void __launch_bounds__(kVoteWarps * 32) classify_kernel(
    const uint32_t* __restrict__ counts, int n_images, int n_exc, const int32_t* __restrict__ labels, int n_classes,
    int32_t* __restrict__ pred) {
  __shared__ unsigned long long s_M[kMaxClasses];
  __shared__ unsigned long long s_sum[kVoteWarps][kMaxClasses];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int c = threadIdx.x; c < n_classes; c += blockDim.x) s_M[c] = 0;
  for (int c = lane; c < n_classes; c += 32) s_sum[warp][c] = 0;
  __syncthreads();
  for (int j = threadIdx.x; j < n_exc; j += blockDim.x) {
    const int l = labels[j];
    if (l >= 0) atomicAdd(&s_M[l], 1ull);
  }
  __syncthreads();
  const int k = blockIdx.x * kVoteWarps + warp;
  if (k >= n_images) return;
  const uint32_t* ck = counts + (size_t)k * n_exc;
  for (int j = lane; j < n_exc; j += 32) {
    const uint32_t x = __ldg(&ck[j]);
    const int l = __ldg(&labels[j]);
    if (x && l >= 0) atomicAdd(&s_sum[warp][l], (unsigned long long)x);
  }
  __syncwarp();
  if (lane == 0) {
    int best = -1;
    for (int c = 0; c < n_classes; ++c) {
      if (s_M[c] == 0 || s_sum[warp][c] == 0) continue;
      if (best < 0 || ratio_gt(s_sum[warp][c], s_M[c], s_sum[warp][best], s_M[best])) best = c;
    }
    pred[k] = best;
  }
}

// ---------------------------------------------------------------- host side
size_t infer_smem_bytes(int R, int row_bytes) {
  return (size_t)R * row_bytes + (size_t)R * 8 + 2 * kSR * 4 + 32 * 8 + 32 * 4 + 2 * kWB * 32 * 4 + 16;
}

template <int BITS, bool FIXED, int MINB>
static cudaError_t launch_infer_t(const InferDesc& d, int grid, int nthr, size_t smem, cudaStream_t s) {
  auto k = infer_kernel<BITS, FIXED, MINB>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k<<<grid, nthr, smem, s>>>(d);
  return cudaGetLastError();
}

template <int BITS, bool FIXED, int MINB>
static cudaError_t occ_t(int nthr, size_t smem, int* out) {
  auto k = infer_kernel<BITS, FIXED, MINB>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(out, k, nthr, smem);
}

// minb: register budget variant (2 -> <= 128 registers, 3 -> <= 80 registers per thread)
cudaError_t infer_occupancy(int bits, int fixed, int minb, int nthr, size_t smem, int* out) {
  switch ((bits * 2 + fixed) * 4 + minb) {
    case 18: return occ_t<2, false, 2>(nthr, smem, out);
    case 19: return occ_t<2, false, 3>(nthr, smem, out);
    case 22: return occ_t<2, true, 2>(nthr, smem, out);
    case 23: return occ_t<2, true, 3>(nthr, smem, out);
    case 34: return occ_t<4, false, 2>(nthr, smem, out);
    case 35: return occ_t<4, false, 3>(nthr, smem, out);
    case 38: return occ_t<4, true, 2>(nthr, smem, out);
    case 39: return occ_t<4, true, 3>(nthr, smem, out);
    case 66: return occ_t<8, false, 2>(nthr, smem, out);
    case 67: return occ_t<8, false, 3>(nthr, smem, out);
    case 70: return occ_t<8, true, 2>(nthr, smem, out);
    case 71: return occ_t<8, true, 3>(nthr, smem, out);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_infer(const InferDesc& d, int grid, int nthr, size_t smem, int fixed, int minb, cudaStream_t s) {
  if (d.n_images <= 0 || d.T <= 0) return cudaSuccess;
  switch ((d.bits * 2 + fixed) * 4 + minb) {
    case 18: return launch_infer_t<2, false, 2>(d, grid, nthr, smem, s);
    case 19: return launch_infer_t<2, false, 3>(d, grid, nthr, smem, s);
    case 22: return launch_infer_t<2, true, 2>(d, grid, nthr, smem, s);
    case 23: return launch_infer_t<2, true, 3>(d, grid, nthr, smem, s);
    case 34: return launch_infer_t<4, false, 2>(d, grid, nthr, smem, s);
    case 35: return launch_infer_t<4, false, 3>(d, grid, nthr, smem, s);
    case 38: return launch_infer_t<4, true, 2>(d, grid, nthr, smem, s);
    case 39: return launch_infer_t<4, true, 3>(d, grid, nthr, smem, s);
    case 66: return launch_infer_t<8, false, 2>(d, grid, nthr, smem, s);
    case 67: return launch_infer_t<8, false, 3>(d, grid, nthr, smem, s);
    case 70: return launch_infer_t<8, true, 2>(d, grid, nthr, smem, s);
    case 71: return launch_infer_t<8, true, 3>(d, grid, nthr, smem, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_pack_infer(const uint8_t* codes, int n_in, int n_exc, int bits, int wpr, uint32_t* w,
                              cudaStream_t s) {
  const size_t n = (size_t)n_in * wpr;
  pack_infer_kernel<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(codes, n_in, n_exc, bits, wpr, w);
  return cudaGetLastError();
}

cudaError_t launch_label(const uint32_t* counts, int n_images, int n_exc, const int32_t* classes, int n_classes,
                         int32_t* labels, cudaStream_t s) {
  label_kernel<<<(unsigned)((n_exc + 127) / 128), 128, 0, s>>>(counts, n_images, n_exc, classes, n_classes, labels);
  return cudaGetLastError();
}

cudaError_t launch_classify(const uint32_t* counts, int n_images, int n_exc, const int32_t* labels, int n_classes,
                            int32_t* pred, cudaStream_t s) {
  if (n_images <= 0) return cudaSuccess;
  classify_kernel<<<(unsigned)((n_images + kVoteWarps - 1) / kVoteWarps), kVoteWarps * 32, 0, s>>>(
      counts, n_images, n_exc, labels, n_classes, pred);
  return cudaGetLastError();
}

}  // namespace snn
