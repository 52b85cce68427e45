// snn_kernels.cu -- sm_100a kernels of the simulate-and-learn loop.
//
// present_kernel: ONE persistent launch presents a whole batch of images (and, for ensembles,
// many independent networks).  Each network is owned by a thread-block cluster of `cs` CTAs;
// CTA r keeps its slice of quantised weight columns resident in shared memory for the whole
// launch (HBM is touched only to load/store the slice once per launch).  Per timestep t:
//   (a1) Philox-keyed Bernoulli encode of the 784 pixels, packed to bits with warp shuffles
//   (a1) compaction of the active input rows (popc / shfl prefix / ffs) + spike timers
//   (a2) integration: one thread per column sums the 2/4/8-bit codes of the active rows (SMEM)
//   (a3) LIF (explicit fmaf or Q15.16 recipe) + refractory / inhibition countdown (registers)
//   (a4) WTA: warp REDUX max of a u64 key -> CTA key -> DSMEM store into every CTA of the
//        cluster -> barrier.cluster (arrive ... wait); LTD, which does not depend on the
//        winner, runs between arrive and wait
//   (a5) LTP (or the deterministic arm, a6) on the winner's column, rows spread over threads
// Citations: P:<line> of /root/reference/PAPER.md; readings R<n> of DESIGN.md §2.
#include "snn_internal.h"
#include "snn_device.cuh"
#include <cstdint>

namespace snn {

struct SmemLayout {
  size_t enc, wkey, slots, w, pot, dep, dbp, dbd, dtp, dtd, lpre, spk, misc, alist, splist, img, total;
};

__host__ __device__ inline SmemLayout smem_layout(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr) {
  SmemLayout L;
  size_t o = 0;
  const int nwi = (n_in + 31) / 32;
  L.enc = o;    o = align16(o + 256 * 8);
  L.wkey = o;   o = align16(o + 32 * 8);
  L.slots = o;  o = align16(o + 2 * kMaxCluster * 8);
  L.w = o;      o = align16(o + (size_t)slice_words * 4);
  L.pot = o;    o = align16(o + (size_t)(L_pot > 0 ? L_pot : 1) * 4);
  L.dep = o;    o = align16(o + (size_t)(L_dep > 0 ? L_dep : 1) * 4);
  const size_t ntab = q_max < 256 ? (size_t)(q_max + 1) : 1;   // 16-bit tables stay in global memory (L2)
  L.dbp = o;    o = align16(o + ntab * 4);
  L.dbd = o;    o = align16(o + ntab * 4);
  L.dtp = o;    o = align16(o + ntab * 4);
  L.dtd = o;    o = align16(o + ntab * 4);
  L.lpre = o;   o = align16(o + (size_t)n_in * 4);
  L.spk = o;    o = align16(o + (size_t)nwi * 4);
  L.misc = o;   o = align16(o + 16 * 4);
  L.alist = o;  o = align16(o + (size_t)n_in * 2);
  L.splist = o; o = align16(o + (size_t)nthr * 2);
  L.img = o;    o = align16(o + (size_t)n_in);
  L.total = o;
  return L;
}

size_t present_smem_bytes(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr) {
  return smem_layout(n_in, slice_words, L_pot, L_dep, q_max, nthr).total;
}

__device__ __forceinline__ int slice_words_of(const NetDesc& d) { return d.slice_words; }

// ---- 32-bit floating-point conductance (bits = 32, NEXT-2, R28); every operation an IEEE-rounded
// intrinsic so that nvcc contracts nothing and the result equals R28's recipe bit for bit
constexpr double kInvLn2 = 0x1.71547652b82fep+0;   // 1/ln 2
constexpr double kLn2Hi = 0x1.62e42feep-1;         // Cody-Waite split of ln 2 (11 trailing zero bits)
constexpr double kLn2Lo = 0x1.a39ef35793c76p-33;

// e^y: y = k ln2 + r (k = rint(y / ln2), two fused multiply-adds), e^r by the degree-kExpDeg Taylor polynomial
// in Horner form (coefficients 1/m! built on the host), times 2^k
__device__ __noinline__ double exp_r28(const NetDesc& d, double y) {
  const double k = rint(__dmul_rn(y, kInvLn2));
  double r = __fma_rn(-k, kLn2Hi, y);
  r = __fma_rn(-k, kLn2Lo, r);
  double e = d.ecoef[kExpDeg];
#pragma unroll
  for (int m = kExpDeg - 1; m >= 0; --m) e = __fma_rn(e, r, d.ecoef[m]);
  return scalbn(e, (int)k);
}

// eqs.(4)(5) P:84 at binary32 G, in binary64: dG_p = alpha_p e^{((-beta_p)(G - G_min)) / (G_max - G_min)},
// dG_d = alpha_d e^{((-beta_d)(G_max - G)) / (G_max - G_min)}
__device__ __forceinline__ double dg_r28(const NetDesc& d, bool depress, float G) {
  const double span = __dsub_rn(d.g_max, d.g_min);
  const double Gd = (double)G;
  if (!depress) return __dmul_rn(d.alpha_p, exp_r28(d, __ddiv_rn(__dmul_rn(-d.beta_p, __dsub_rn(Gd, d.g_min)), span)));
  return __dmul_rn(d.alpha_d, exp_r28(d, __ddiv_rn(__dmul_rn(-d.beta_d, __dsub_rn(d.g_max, Gd)), span)));
}

// G' = binary32(G +- dG) (binary64 add, one rounding to nearest), clamped to [G_min, G_max]
__device__ __forceinline__ uint32_t gstep_r28(const NetDesc& d, uint32_t word, bool depress) {
  const float G = __uint_as_float(word);
  const double dG = dg_r28(d, depress, G);
  float G1 = __double2float_rn(depress ? __dsub_rn((double)G, dG) : __dadd_rn((double)G, dG));
  G1 = G1 < d.gminf ? d.gminf : G1;
  G1 = G1 > d.gmaxf ? d.gmaxf : G1;
  return __float_as_uint(G1);
}

// ------------------------------------------------------------------ the persistent step kernel
__global__ void __launch_bounds__(kMaxThreads, 1) present_kernel(const __grid_constant__ LaunchParams lp) {
  extern __shared__ __align__(16) unsigned char smem[];
  const NetDesc& d0 = lp.descs ? lp.descs[0] : lp.single;
  const int cs = d0.cs;
  const int net = blockIdx.x / cs;
  const int rank = blockIdx.x - net * cs;           // == %cluster_ctarank for 1-D clusters
  const NetDesc& d = lp.descs ? lp.descs[net] : lp.single;

  const int n_in = d.n_in, n_exc = d.n_exc, bits = d.bits, qmax = d.q_max, wpr = d.wpr;
  const int nwi = d.nwi, nwe = d.nwe, T = d.T, flags = d.flags;
  const int L_pot = d.L_pot, L_dep = d.L_dep;
  const int slice_words = slice_words_of(d);
  const SmemLayout L = smem_layout(n_in, slice_words, L_pot, L_dep, qmax, blockDim.x);
  unsigned long long* s_enc = reinterpret_cast<unsigned long long*>(smem + L.enc);
  unsigned long long* s_wkey = reinterpret_cast<unsigned long long*>(smem + L.wkey);
  unsigned long long* s_slots = reinterpret_cast<unsigned long long*>(smem + L.slots);
  uint32_t* s_w = reinterpret_cast<uint32_t*>(smem + L.w);
  uint32_t* s_pot = reinterpret_cast<uint32_t*>(smem + L.pot);
  uint32_t* s_dep = reinterpret_cast<uint32_t*>(smem + L.dep);
  const bool tab_smem = d.q_max < 256;
  const int* s_dbp = tab_smem ? reinterpret_cast<const int*>(smem + L.dbp) : d.det_base_p;
  const int* s_dbd = tab_smem ? reinterpret_cast<const int*>(smem + L.dbd) : d.det_base_d;
  const uint32_t* s_dtp = tab_smem ? reinterpret_cast<const uint32_t*>(smem + L.dtp) : d.det_thr_p;
  const uint32_t* s_dtd = tab_smem ? reinterpret_cast<const uint32_t*>(smem + L.dtd) : d.det_thr_d;
  int* s_lpre = reinterpret_cast<int*>(smem + L.lpre);
  uint32_t* s_spk = reinterpret_cast<uint32_t*>(smem + L.spk);
  int* s_misc = reinterpret_cast<int*>(smem + L.misc);
  uint16_t* s_alist = reinterpret_cast<uint16_t*>(smem + L.alist);
  uint16_t* s_splist = reinterpret_cast<uint16_t*>(smem + L.splist);
  uint8_t* s_img = smem + L.img;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nthr = blockDim.x;
  // column slice of this CTA: groups [g0, g1) of 32 columns
  const int g0 = (rank * d.ngroups) / cs, g1 = ((rank + 1) * d.ngroups) / cs;
  const int col0 = g0 * 32;
  const int ncols = min(g1 * 32, n_exc) - col0;
  const int ngrp_cta = g1 - g0;
  const bool mycol = tid < ncols;
  const int j = col0 + tid;                          // this CTA-slice column (state arrays are per shard)
  // column sharding: this network is columns [col_base, col_base + n_exc) of a network split over
  // `world` ranks; every random draw and WTA key uses GLOBAL column indices, and per step the clusters' WTA summaries
  // meet in every rank's mailbox, so the union of the shards is the unsharded network bit for bit
  const int cbase = d.col_base;
  const int jg = cbase + j;                          // global column
  const int world = d.world;
  const bool sharded = world > 1;
  const uint32_t seq0 = sharded ? (uint32_t)ld_relaxed_sys_s32(reinterpret_cast<const int*>(&d.mbox->seq)) : 0u;
  uint32_t nxch = 0;                                 // exchanges of this launch (one per step)
  const int lg = bits == 2 ? 4 : (bits == 4 ? 3 : (bits == 8 ? 2 : (bits == 16 ? 1 : 0)));   // log2(codes per word)
  const int wj = tid >> lg;
  const int sh = (tid & ((1 << lg) - 1)) * bits;
  const uint32_t fmask = bits == 32 ? 0xFFFFFFFFu : (1u << bits) - 1u;
  const bool wide = bits > 8;       // 16-bit codes: STDP steps by eqs.(4)(5) magnitudes, not 1 LSB (R27)
  const bool f32 = bits == 32;      // binary32 conductance, one column per word (R28)
  const int nq4 = (n_in + 3) >> 2;
  const bool fixed = d.membrane_mode == 1;
  const bool hard = d.wta_mode == 0;
  const bool stoch = d.stdp_mode == 0;
  const bool inh_reset = d.inh_mode == 0;
  const bool floor_mode = (flags & FLAG_FLOOR) != 0;   // bench: same launch shape, barriers + exchange only
  const bool learn = (flags & FLAG_NO_LEARN) == 0;     // inference (R21): steps 1-4 only, weights and state kept

  // ---- one-time staging: tables + this CTA's weight slice -> SMEM
  for (int k = tid; k < 256; k += nthr) s_enc[k] = d.thr_enc[k];
  for (int k = tid; k < L_pot; k += nthr) s_pot[k] = d.pot_m1[k];
  for (int k = tid; k < L_dep; k += nthr) s_dep[k] = d.dep_m1[k];
  if (tab_smem)
    for (int k = tid; k <= qmax; k += nthr) {
      const_cast<int*>(s_dbp)[k] = d.det_base_p[k]; const_cast<int*>(s_dbd)[k] = d.det_base_d[k];
      const_cast<uint32_t*>(s_dtp)[k] = d.det_thr_p[k];  const_cast<uint32_t*>(s_dtd)[k] = d.det_thr_d[k];
    }
  {
    const uint4* src = reinterpret_cast<const uint4*>(d.wslices + (size_t)rank * slice_words);
    uint4* dst = reinterpret_cast<uint4*>(s_w);
    for (int k = tid; k < slice_words / 4; k += nthr) dst[k] = src[k];
  }
  int v_r = fixed ? d.Vinit : __float_as_int(d.vinitf);
  int cnt_r = 0, lpost_r = kNever;
  const bool keep = (flags & FLAG_KEEP_STATE) != 0;
  if (keep) {
    if (mycol) { v_r = d.v[j]; cnt_r = d.cnt[j]; lpost_r = d.last_post[j]; }
    for (int i = tid; i < n_in; i += nthr) s_lpre[i] = d.last_pre[i];
  }
  uint32_t ltd_trials = 0, ltd_events = 0, ltp_trials = 0, ltp_events = 0;
  unsigned long long act_sum = 0, post_sum = 0;
  // every CTA of the cluster must have started before another addresses its shared memory (DSMEM stores below)
  if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }

  for (int b = 0; b < d.n_images; ++b) {
    const unsigned long long seed = d.seeds[b];
    const int t0 = keep ? d.t0 : 0;
    if (!keep) {                                              // R5: per-presentation reset
      v_r = fixed ? d.Vinit : __float_as_int(d.vinitf);
      cnt_r = 0; lpost_r = kNever;
      for (int i = tid; i < n_in; i += nthr) s_lpre[i] = kNever;
    }
    if (!(flags & FLAG_RASTER_INPUT))
      for (int i = tid; i < n_in; i += nthr) s_img[i] = d.images[(size_t)b * n_in + i];
    const bool last_img = (b == d.n_images - 1);
    const bool rec_in = last_img && rank == 0 && d.in_raster_out != nullptr;
    const bool rec_out = last_img && d.raster_out != nullptr;
    int img_spikes = 0;
    uint32_t ncount = 0;                                      // this column's spikes in the image (inference)
    __syncthreads();

    for (int k = 0; k < T; ++k) {
      const int t = t0 + k;
      const int par = k & 1;

      // (a1) ENCODE: s_i = u_ENC(t, i) < thr_enc[x_i]   (R8, R13)
      if (floor_mode) {
        for (int w = tid; w < nwi; w += nthr) s_spk[w] = 0u;
      } else if (flags & FLAG_RASTER_INPUT) {
        for (int w = tid; w < nwi; w += nthr) s_spk[w] = d.in_raster[(size_t)k * nwi + w];
      } else {
        for (int base = warp * 32; base < nq4; base += nthr) {     // warp-uniform trip count
          const int q = base + lane;
          uint32_t nib = 0;
          if (q < nq4) {
            const uint4 u = philox((uint32_t)t, (uint32_t)q, 0u, TAG_ENC, seed);
#pragma unroll
            for (int r = 0; r < 4; ++r) {
              const int i = 4 * q + r;
              if (i < n_in && (unsigned long long)pick(u, r) < s_enc[s_img[i]]) nib |= 1u << r;
            }
          }
          uint32_t x = nib << (4 * (lane & 7));
          x |= __shfl_xor_sync(FULL, x, 1);
          x |= __shfl_xor_sync(FULL, x, 2);
          x |= __shfl_xor_sync(FULL, x, 4);
          const int w = q >> 3;
          if ((lane & 7) == 0 && w < nwi) s_spk[w] = x;
        }
      }
      __syncthreads();                                                         // B1

      // (a1) active rows, ascending; spike timers last_pre
      if (warp == 0) {
        int base = 0;
        for (int w0 = 0; w0 < nwi; w0 += 32) {
          const int w = w0 + lane;
          uint32_t word = w < nwi ? s_spk[w] : 0u;
          if (rec_in && w < nwi) d.in_raster_out[(size_t)k * nwi + w] = word;
          const int c = __popc(word);
          int incl = c;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
          }
          int pos = base + incl - c;
          while (word) {
            const int bp = __ffs(word) - 1;
            word &= word - 1;
            const int i = w * 32 + bp;
            s_alist[pos++] = (uint16_t)i;
            s_lpre[i] = t;
          }
          base += __shfl_sync(FULL, incl, 31);
        }
        if (lane == 0) { s_misc[0] = base; s_misc[1] = 0; }
      }
      __syncthreads();                                                         // B2
      const int nact = s_misc[0];
      if (rank == 0 && tid == 0) act_sum += (unsigned long long)nact;

      // (a2) INTEGRATE eq.(3): S_j = sum_{active i} q_ij      (a3) LIF eqs.(1)(2)
      bool cand = false;
      if (mycol && !floor_mode) {
        int S = 0;
        float Sg = 0.0f;                                   // R28: binary32 sum, ascending rows, from +0
        const uint32_t* wcol = s_w + wj;
        if (f32)
          for (int a = 0; a < nact; ++a) Sg = __fadd_rn(Sg, __uint_as_float(wcol[(int)s_alist[a] * wpr]));
        else
          for (int a = 0; a < nact; ++a) S += (int)((wcol[(int)s_alist[a] * wpr] >> sh) & fmask);
        if (cnt_r > 0) {
          --cnt_r;
        } else if (fixed) {
          const long long v = v_r;
          const long long bv = (d.B * v + (1LL << 31)) >> 32;
          const long long cterm = (d.C * (long long)S + (1LL << 15)) >> 16;
          v_r = (int)(v + d.A + bv + cterm + d.E);
          cand = v_r > d.Vth;
        } else {
          const float vf = __int_as_float(v_r);
          const float I = f32 ? __fmul_rn(Sg, d.kV) : __fmul_rn(__int2float_rn(S), d.kI);
          const float x = __fadd_rn(I, d.ief);
          const float y = __fmaf_rn(d.cf, x, d.af);
          const float dv = __fmaf_rn(d.bf, vf, y);
          const float vn = __fmaf_rn(d.dtf, dv, vf);
          v_r = __float_as_int(vn);
          cand = vn > d.vthf;
        }
      }

      // (a4) WTA, CTA level (R7): HARD -> max key (ord(v) << 32 | ~j);  LAYER -> candidate count
      unsigned long long ctakey = 0;
      int cta_count = 0;
      if (hard) {
        uint32_t ord = 0, lo = 0;
        if (cand) {
          ord = fixed ? ((uint32_t)v_r ^ 0x80000000u) : float_ord((uint32_t)v_r);
          lo = 0xFFFFFFFFu - (uint32_t)jg;
        }
        const uint32_t mh = __reduce_max_sync(FULL, ord);
        const uint32_t ml = __reduce_max_sync(FULL, ord == mh ? lo : 0u);
        if (lane == 0) s_wkey[warp] = ((unsigned long long)mh << 32) | ml;
        cta_count = __syncthreads_or(cand);                                    // B3
        if (warp == 0 && cta_count) {
          const unsigned long long kk = lane < (nthr >> 5) ? s_wkey[lane] : 0ull;
          const uint32_t h = (uint32_t)(kk >> 32), l = (uint32_t)kk;
          const uint32_t mh2 = __reduce_max_sync(FULL, h);
          const uint32_t ml2 = __reduce_max_sync(FULL, h == mh2 ? l : 0u);
          ctakey = ((unsigned long long)mh2 << 32) | ml2;
        }
      } else {
        cta_count = __syncthreads_count(cand);                                 // B3
        ctakey = (unsigned long long)cta_count;
      }
      // publish the CTA's candidate to slot[par][rank] of every CTA of the cluster
      if (warp == 0) {
        if (cs == 1) {
          if (lane == 0) s_slots[par * kMaxCluster] = ctakey;
        } else if (lane < cs) {
          st_cluster_u64(&s_slots[par * kMaxCluster + rank], (uint32_t)lane, ctakey);
        }
      }
      if (cs > 1) cluster_arrive();

      // (a5) LTD, overlapped with the exchange: pre spikes at t against last_post (eq.(7), R10, R14).
      // Column-local and independent of this step's winner (uses the old last_post).
      if (learn && stoch && mycol && lpost_r >= 0) {
        const int D = t - lpost_r;
        if (D < L_dep) {
          const uint32_t thr = s_dep[D];
          uint32_t* wcol = s_w + wj;
          for (int a = 0; a < nact; ++a) {
            const int i = s_alist[a];
            const uint4 u = philox((uint32_t)t, (uint32_t)i, (uint32_t)(jg >> 2), TAG_LTD, seed);
            ++ltd_trials;
            if (pick(u, jg & 3) <= thr) {
              ++ltd_events;
              uint32_t* p = wcol + i * wpr;
              if (f32) {                                        // eq.(5) in binary32 (R28); own word
                *p = gstep_r28(d, *p, true);
              } else if (!wide) {
                if ((*p >> sh) & fmask) atomicSub(p, 1u << sh);   // other fields of the word may move concurrently
              } else {                                          // eq.(5) rounded (eq.(8), R27)
                const int q0 = (int)((*p >> sh) & fmask);
                const uint4 u2 = philox((uint32_t)t, (uint32_t)i, (uint32_t)(jg >> 2), TAG_ROUND_LTD, seed);
                const int dq = s_dbd[q0] + (pick(u2, jg & 3) < s_dtd[q0] ? 1 : 0);
                const int q1 = q0 - dq < 0 ? 0 : q0 - dq;
                if (q1 != q0) atomicSub(p, (uint32_t)(q0 - q1) << sh);   // only this thread moves this field
              }
            }
          }
        }
      }
      if (cs > 1) cluster_wait(); else __syncthreads();                        // B4 / cluster barrier

      // global decision
      int W = -1, total = 0;
      unsigned long long m = 0;                       // HARD: the cluster's best key; LAYER: its spiker count
      if (hard) {
        for (int r = 0; r < cs; ++r) { const unsigned long long x = s_slots[par * kMaxCluster + r]; m = x > m ? x : m; }
      } else {
        for (int r = 0; r < cs; ++r) m += s_slots[par * kMaxCluster + r];
      }
      if (sharded) {
        // the cluster's value goes to slot [cur & 1][shard] of every rank's mailbox as two LL words (peer stores, no
        // fence); warp 0 of every CTA polls its own mailbox for the world's values and applies the same reduction
        const uint32_t cur = seq0 + ++nxch;
        const int mp = (int)(cur & 1u);
        const unsigned long long tag = (unsigned long long)cur << 32;
        if (rank == 0 && warp == 0 && lane < world) {
          unsigned long long* sl = d.peers[lane]->slot[mp][d.shard];
          st_relaxed_sys_u64(sl, tag | (uint32_t)(m >> 32));
          st_relaxed_sys_u64(sl + 1, tag | (uint32_t)m);
        }
        if (warp == 0) {
          unsigned long long x = 0ull;
          if (lane < world) {
            const unsigned long long* sl = d.mbox->slot[mp][lane];
            const unsigned long long t_start = globaltimer();
            unsigned long long w0, w1;
            while (true) {
              w0 = ld_relaxed_sys_u64(sl); w1 = ld_relaxed_sys_u64(sl + 1);
              if ((uint32_t)(w0 >> 32) == cur && (uint32_t)(w1 >> 32) == cur) break;
              if (globaltimer() - t_start > kShardTimeoutNs) __trap();   // a rank is gone: fail, never hang
            }
            x = ((unsigned long long)(uint32_t)w0 << 32) | (uint32_t)w1;
          }
          const uint32_t xh = (uint32_t)(x >> 32), xl = (uint32_t)x;
          unsigned long long g;
          if (hard) {
            const uint32_t mh = __reduce_max_sync(FULL, xh);
            g = ((unsigned long long)mh << 32) | __reduce_max_sync(FULL, xh == mh ? xl : 0u);
          } else {
            g = __reduce_add_sync(FULL, xl);
          }
          if (lane == 0) s_misc[8 + par * 2] = (int)(uint32_t)(g >> 32), s_misc[9 + par * 2] = (int)(uint32_t)g;
        }
        __syncthreads();
        m = ((unsigned long long)(uint32_t)s_misc[8 + par * 2] << 32) | (uint32_t)s_misc[9 + par * 2];
      }
      if (hard) {
        if (m) W = (int)(0xFFFFFFFFu - (uint32_t)m);     // global column
      } else {
        total = (int)m;
      }

      // apply eq.(2) reset, refractory, lateral inhibition (R6, R7)
      bool spiked = false;
      bool local_spike = false;
      if (hard) {
        if (W >= 0) {
          if (mycol) {
            if (jg == W) { v_r = fixed ? d.Vreset : __float_as_int(d.vresetf); cnt_r = d.t_ref; spiked = true; }
            else {
              cnt_r = max(cnt_r, d.t_inh);
              if (inh_reset) v_r = fixed ? d.Vreset : __float_as_int(d.vresetf);
            }
          }
          img_spikes += 1;
          local_spike = (W >= cbase + col0 && W < cbase + col0 + ncols);
        }
      } else if (total > 0) {
        if (mycol) {
          if (cand) { v_r = fixed ? d.Vreset : __float_as_int(d.vresetf); cnt_r = d.t_ref; spiked = true; }
          if (total >= 2 || !cand) {
            cnt_r = max(cnt_r, d.t_inh);
            if (inh_reset) v_r = fixed ? d.Vreset : __float_as_int(d.vresetf);
          }
        }
        img_spikes += total;
        local_spike = cta_count > 0;
        if (spiked) { const int pos = atomicAdd(&s_misc[1], 1); s_splist[pos] = (uint16_t)tid; }
      }
      if (rec_out) {
        const uint32_t bal = __ballot_sync(FULL, spiked);
        if (lane == 0 && warp < ngrp_cta) d.raster_out[(size_t)k * nwe + g0 + warp] = bal;
      }
      if (spiked) ++ncount;

      // (a5) LTP (eq.(6)) or (a6) the deterministic arm (eqs.(4)(5)(8)) on the spiking columns.
      // Thread g owns input rows 4g..4g+3 (their words), so no atomics are needed here.
      if (local_spike && learn) {
        __syncthreads();                                                       // B5: LTD done, splist built
        const int nsp = hard ? 1 : s_misc[1];
        for (int grp = tid; grp < nq4; grp += nthr) {
          for (int m = 0; m < nsp; ++m) {
            const int Wl = hard ? (W - cbase - col0) : (int)s_splist[m];
            const int Wg = cbase + col0 + Wl;
            const int ww = Wl >> lg, wsh = (Wl & ((1 << lg) - 1)) * bits;
            const uint4 u = philox((uint32_t)t, (uint32_t)Wg, (uint32_t)grp, stoch ? TAG_LTP : TAG_ROUND, seed);
#pragma unroll
            for (int r = 0; r < 4; ++r) {
              const int i = 4 * grp + r;
              if (i >= n_in) break;
              const int lp = s_lpre[i];
              uint32_t* p = s_w + i * wpr + ww;
              if (stoch) {
                if (lp < 0) continue;
                const int D = t - lp;
                if (D >= L_pot) continue;
                ++ltp_trials;
                if (pick(u, r) <= s_pot[D]) {
                  ++ltp_events;
                  const uint32_t word = *p;
                  const int q0 = (int)((word >> wsh) & fmask);
                  if (f32) {                                // eq.(4) in binary32 (R28)
                    *p = gstep_r28(d, word, false);
                  } else if (!wide) {
                    if (q0 < qmax) *p = word + (1u << wsh);
                  } else {                                  // eq.(4) rounded (eq.(8), R27)
                    const uint4 u2 = philox((uint32_t)t, (uint32_t)Wg, (uint32_t)grp, TAG_ROUND, seed);
                    const int dq = s_dbp[q0] + (pick(u2, r) < s_dtp[q0] ? 1 : 0);
                    const int q1 = q0 + dq > qmax ? qmax : q0 + dq;
                    *p = (word & ~(fmask << wsh)) | ((uint32_t)q1 << wsh);
                  }
                }
              } else if (f32) {                             // R16 window, eqs.(4)(5) in binary32 (R28)
                const bool pot = lp >= 0 && (t - lp) <= d.t_ltp;
                const float G = __uint_as_float(*p);
                *p = gstep_r28(d, *p, !pot);
                if (dg_r28(d, !pot, G) > 0.0) { if (pot) ++ltp_events; else ++ltd_events; }
                if (pot) ++ltp_trials; else ++ltd_trials;
              } else {
                const uint32_t word = *p;
                const int q0 = (int)((word >> wsh) & fmask);
                const bool pot = lp >= 0 && (t - lp) <= d.t_ltp;
                const int base = pot ? s_dbp[q0] : s_dbd[q0];
                const uint32_t thr = pot ? s_dtp[q0] : s_dtd[q0];
                const int dq = base + (pick(u, r) < thr ? 1 : 0);
                int q1 = pot ? q0 + dq : q0 - dq;
                q1 = q1 < 0 ? 0 : (q1 > qmax ? qmax : q1);
                *p = (word & ~(fmask << wsh)) | ((uint32_t)q1 << wsh);
                if (pot) { ++ltp_trials; if (dq > 0) ++ltp_events; }
                else     { ++ltd_trials; if (dq > 0) ++ltd_events; }
              }
            }
          }
        }
      }
      if (spiked) lpost_r = t;                                                 // spike timer
    }  // steps

    if (rank == 0 && tid == 0) {
      post_sum += (unsigned long long)img_spikes;
      if (d.spike_counts) d.spike_counts[b] = img_spikes;
    }
    if (d.neuron_counts && mycol) d.neuron_counts[(size_t)b * n_exc + j] = ncount;
    if (last_img && learn) {
      if (mycol) { d.v[j] = v_r; d.cnt[j] = cnt_r; d.last_post[j] = lpost_r; }
      if (rank == 0) for (int i = tid; i < n_in; i += nthr) d.last_pre[i] = s_lpre[i];
    }
    __syncthreads();
  }  // images

  // write the (learned) slice back to HBM
  if (learn) {
    uint4* dst = reinterpret_cast<uint4*>(d.wslices + (size_t)rank * slice_words);
    const uint4* src = reinterpret_cast<const uint4*>(s_w);
    for (int k = tid; k < slice_words / 4; k += nthr) dst[k] = src[k];
  }
  // counters (R20)
  {
    unsigned long long a = ltd_trials, b2 = ltd_events, c = ltp_trials, e = ltp_events;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      a += __shfl_xor_sync(FULL, a, o); b2 += __shfl_xor_sync(FULL, b2, o);
      c += __shfl_xor_sync(FULL, c, o); e += __shfl_xor_sync(FULL, e, o);
    }
    if (lane == 0) {
      if (a) atomicAdd(&d.stats[2], a);
      if (b2) atomicAdd(&d.stats[3], b2);
      if (c) atomicAdd(&d.stats[4], c);
      if (e) atomicAdd(&d.stats[5], e);
    }
    if (rank == 0 && tid == 0) {
      atomicAdd(&d.stats[0], act_sum);
      atomicAdd(&d.stats[1], post_sum);
      atomicAdd(&d.stats[6], (unsigned long long)d.n_images);
      atomicAdd(&d.stats[7], (unsigned long long)d.n_images * (unsigned long long)T);
    }
  }
  if (sharded && rank == 0 && tid == 0) d.mbox->seq = seq0 + nxch;   // every CTA read seq0 long ago
  if (cs > 1) { cluster_arrive(); cluster_wait(); }   // no CTA leaves while peers may address its SMEM
}

cudaError_t configure_present_kernel(size_t smem, int cs) {
  cudaError_t e = cudaFuncSetAttribute(present_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (cs > 8) e = cudaFuncSetAttribute(present_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  return e;
}

static void fill_cfg(cudaLaunchConfig_t& cfg, cudaLaunchAttribute* attr, int n_nets, int cs, int nthr, size_t smem,
                     cudaStream_t s) {
  cfg = cudaLaunchConfig_t{};
  cfg.gridDim = dim3((unsigned)(n_nets * cs));
  cfg.blockDim = dim3((unsigned)nthr);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.numAttrs = 0;
  cfg.attrs = attr;
  if (cs > 1) {
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.numAttrs = 1;
  }
}

cudaError_t query_max_clusters(int cs, int nthr, size_t smem, int* out) {
  cudaError_t e = configure_present_kernel(smem, cs);
  if (e != cudaSuccess) return e;
  if (cs == 1) {
    int nb = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, present_kernel, nthr, smem);
    *out = nb;
    return e;
  }
  cudaLaunchConfig_t cfg;
  cudaLaunchAttribute attr[1];
  fill_cfg(cfg, attr, 1, cs, nthr, smem, 0);
  return cudaOccupancyMaxActiveClusters(out, present_kernel, &cfg);
}

cudaError_t launch_present(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, cudaStream_t s) {
  cudaError_t e = configure_present_kernel(smem, cs);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg;
  cudaLaunchAttribute attr[1];
  fill_cfg(cfg, attr, n_nets, cs, nthr, smem, s);
  return cudaLaunchKernelEx(&cfg, present_kernel, lp);
}

// ------------------------------------------------------------------ weight layout kernels
// One thread per packed word (rank r, row i, word w) of the slice image [cs][n_in][wpr].
__device__ __forceinline__ bool word_coords(const NetDesc& d, size_t gid, int& r, int& i, int& w, int& col0,
                                            int& ncols) {
  const int sw = slice_words_of(d);
  const size_t total = (size_t)d.cs * sw;
  if (gid >= total) return false;
  r = (int)(gid / sw);
  const int rem = (int)(gid - (size_t)r * sw);
  i = rem / d.wpr;
  w = rem - i * d.wpr;
  if (i >= d.n_in) return false;       // padding words at the end of a slice
  const int g0 = (r * d.ngroups) / d.cs, g1 = ((r + 1) * d.ngroups) / d.cs;
  col0 = g0 * 32;
  ncols = min(g1 * 32, d.n_exc) - col0;
  return true;
}

__global__ void init_weights_kernel(const NetDesc d, unsigned long long init_seed) {
  const size_t gid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  int r, i, w, col0, ncols;
  const int sw = slice_words_of(d);
  if (gid < (size_t)d.cs * sw) d.wslices[gid] = 0u;
  if (!word_coords(d, gid, r, i, w, col0, ncols)) return;
  const int cpw = 32 / d.bits;
  uint32_t word = 0;
  for (int c = 0; c < cpw; ++c) {
    const int jl = w * cpw + c;
    if (jl >= ncols) break;
    const int jg = d.col_base + col0 + jl;                  // global column (a shard starts at col_base)
    const uint4 u = philox((uint32_t)i, (uint32_t)(jg >> 2), 0u, TAG_INIT, init_seed);   // R4
    if (d.bits == 32) {                                     // R28: G = binary32(G_max (u >> 8) 2^-24)
      word = __float_as_uint(__double2float_rn(__dmul_rn(d.g_max, scalbn((double)(pick(u, jg & 3) >> 8), -24))));
      break;
    }
    const uint32_t code = (uint32_t)(((unsigned long long)pick(u, jg & 3) * (unsigned long long)(d.q_max + 1)) >> 32);
    word |= code << (c * d.bits);
  }
  d.wslices[gid] = word;
}

// codes: one byte per code (bits <= 8), one uint16 per code (bits = 16) or the binary32 G (bits = 32, R28),
// row-major [i][j]
__device__ __forceinline__ uint32_t code_at(const NetDesc& d, const void* codes, size_t k) {
  if (d.bits == 32) return static_cast<const uint32_t*>(codes)[k];
  return d.bits > 8 ? (uint32_t)static_cast<const uint16_t*>(codes)[k] : (uint32_t)static_cast<const uint8_t*>(codes)[k];
}
__device__ __forceinline__ uint32_t field_mask(int bits) { return bits == 32 ? 0xFFFFFFFFu : (1u << bits) - 1u; }

__global__ void pack_weights_kernel(const NetDesc d, const void* __restrict__ codes) {
  const size_t gid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  int r, i, w, col0, ncols;
  const int sw = slice_words_of(d);
  if (gid < (size_t)d.cs * sw) d.wslices[gid] = 0u;
  if (!word_coords(d, gid, r, i, w, col0, ncols)) return;
  const int cpw = 32 / d.bits;
  uint32_t word = 0;
  for (int c = 0; c < cpw; ++c) {
    const int jl = w * cpw + c;
    if (jl >= ncols) break;
    word |= (code_at(d, codes, (size_t)i * d.n_exc + col0 + jl) & field_mask(d.bits)) << (c * d.bits);
  }
  d.wslices[gid] = word;
}

__global__ void unpack_weights_kernel(const NetDesc d, void* __restrict__ codes) {
  const size_t gid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  int r, i, w, col0, ncols;
  if (!word_coords(d, gid, r, i, w, col0, ncols)) return;
  const int cpw = 32 / d.bits;
  const uint32_t word = d.wslices[gid];
  for (int c = 0; c < cpw; ++c) {
    const int jl = w * cpw + c;
    if (jl >= ncols) break;
    const uint32_t code = (word >> (c * d.bits)) & field_mask(d.bits);
    const size_t k = (size_t)i * d.n_exc + col0 + jl;
    if (d.bits == 32) static_cast<uint32_t*>(codes)[k] = code;
    else if (d.bits > 8) static_cast<uint16_t*>(codes)[k] = (uint16_t)code;
    else static_cast<uint8_t*>(codes)[k] = (uint8_t)code;
  }
}

__global__ void check_codes_kernel(const void* __restrict__ codes, size_t n, int bits, int q_max, int* bad) {
  const size_t gid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= n) return;
  const int c = bits > 8 ? (int)static_cast<const uint16_t*>(codes)[gid] : (int)static_cast<const uint8_t*>(codes)[gid];
  if (c > q_max) atomicAdd(bad, 1);
}

// R28: every binary32 conductance finite and inside [G_min, G_max] (NaN fails both comparisons)
__global__ void check_g_kernel(const float* __restrict__ g, size_t n, float gmin, float gmax, int* bad) {
  const size_t gid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= n) return;
  const float x = g[gid];
  if (!(x >= gmin && x <= gmax)) atomicAdd(bad, 1);
}

static unsigned grid_for(size_t n, int bs) { return (unsigned)((n + bs - 1) / bs); }

cudaError_t launch_init_weights(const NetDesc& d, uint64_t init_seed, cudaStream_t s) {
  const size_t n = (size_t)d.cs * d.slice_words;
  init_weights_kernel<<<grid_for(n, 256), 256, 0, s>>>(d, init_seed);
  return cudaGetLastError();
}
cudaError_t launch_pack_weights(const NetDesc& d, const void* codes, cudaStream_t s) {
  const size_t n = (size_t)d.cs * d.slice_words;
  pack_weights_kernel<<<grid_for(n, 256), 256, 0, s>>>(d, codes);
  return cudaGetLastError();
}
cudaError_t launch_unpack_weights(const NetDesc& d, void* codes, cudaStream_t s) {
  const size_t n = (size_t)d.cs * d.slice_words;
  unpack_weights_kernel<<<grid_for(n, 256), 256, 0, s>>>(d, codes);
  return cudaGetLastError();
}
cudaError_t launch_check_g(const float* g, size_t n, float gmin, float gmax, int* bad, cudaStream_t s) {
  check_g_kernel<<<grid_for(n, 256), 256, 0, s>>>(g, n, gmin, gmax, bad);
  return cudaGetLastError();
}
cudaError_t launch_check_codes(const void* codes, size_t n, int bits, int q_max, int* bad, cudaStream_t s) {
  check_codes_kernel<<<grid_for(n, 256), 256, 0, s>>>(codes, n, bits, q_max, bad);
  return cudaGetLastError();
}

}  // namespace snn
