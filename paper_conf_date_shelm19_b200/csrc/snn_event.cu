// snn_event.cu -- event-driven engine of the simulate-and-learn loop.
//
// Why: on B200 one cross-SM exchange costs 0.45-0.8 us (barrier.cluster, cs 2..16; profiles/
// r01_sync_probe.txt) while a timestep of one column is ~0.05 us of work.  The per-step engine
// (snn_kernels.cu) pays the exchange every step.  But between two post-synaptic spikes the
// columns of the network are independent: inhibition, LTP and last_post change only at post
// spikes (P:88 WTA, R7, R10), and LTD at step t depends only on the column's own last_post
// and the input spikes (R14).  So each thread runs its column ahead on its own -- integration
// (eq.(3)), LIF (eqs.(1)(2)) and LTD (eq.(7)), exactly -- until its column first crosses the
// threshold; a shared early-stop flag (DSMEM red.min) tells the rest of the cluster where the
// first crossing so far is.  One cluster exchange per EPOCH then fixes the first crossing step
// t* and the winner; threads that ran past t* roll back (RESET inhibition: O(1) state rebuild
// + undo of their logged LTD steps after t*; otherwise re-simulation from the epoch start).
// The result is bit-identical to the per-step semantics (tests/test_gpu_parity.py).
//
// Pre-pass (grid-wide, parallel over images x steps): the Philox encoder (a1) writes bit-packed
// input rasters; a compaction kernel turns them into per-step active-row lists that the main
// kernel stages into shared memory per image.
#include "snn_internal.h"
#include "snn_device.cuh"

#include <climits>
#include <cstdint>

namespace snn {

// ====================================================================== pre-pass 1: encoder (a1)
// one warp per (image, step); lane w builds input word w (32 pixels = 8 Philox blocks)
constexpr int kEncWarps = 4;

__global__ void __launch_bounds__(kEncWarps * 32) encode_kernel(
    const uint8_t* __restrict__ images, const unsigned long long* __restrict__ thr_enc,
    const unsigned long long* __restrict__ seeds, int n_in, int T, int t0, uint32_t* __restrict__ words,
    uint32_t* __restrict__ counts) {
  __shared__ unsigned long long s_thr[256];
  for (int x = threadIdx.x; x < 256; x += blockDim.x) s_thr[x] = thr_enc[x];
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int b = blockIdx.y;
  const int k = blockIdx.x * kEncWarps + warp;
  if (k >= T) return;
  const int nwi = (n_in + 31) >> 5;
  const unsigned long long seed = seeds[b];
  const uint32_t t = (uint32_t)(t0 + k);
  const uint8_t* img = images + (size_t)b * n_in;
  uint32_t* wout = words + ((size_t)b * T + k) * nwi;
  uint32_t c = 0;
  for (int w = lane; w < nwi; w += 32) {
    uint32_t word = 0;
#pragma unroll
    for (int g = 0; g < 8; ++g) {
      const int q = 8 * w + g;
      if (4 * q < n_in) {
        const uint4 u = philox(t, (uint32_t)q, 0u, TAG_ENC, seed);   // (t, i>>2, 0, ENC)[i&3], R13
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          const int i = 4 * q + r;
          if (i < n_in && (unsigned long long)pick(u, r) < s_thr[img[i]]) word |= 1u << (4 * g + r);
        }
      }
    }
    wout[w] = word;
    c += __popc(word);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
  if (lane == 0) counts[(size_t)b * T + k] = c;
}

__global__ void counts_from_raster_kernel(const uint32_t* __restrict__ raster, int n_in, int T, uint32_t* __restrict__ counts) {
  const int lane = threadIdx.x & 31;
  const int k = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (k >= T) return;
  const int nwi = (n_in + 31) >> 5;
  uint32_t c = 0;
  for (int w = lane; w < nwi; w += 32) {
    uint32_t word = raster[(size_t)k * nwi + w];
    if (w == nwi - 1 && (n_in & 31)) word &= (1u << (n_in & 31)) - 1u;
    c += __popc(word);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
  if (lane == 0) counts[k] = c;
}

// ====================================================================== pre-pass 2: compaction
// one CTA per image: exclusive scan of the per-step counts -> offs[T+1]; then one warp per step
// expands the bit-packed words into ascending row indices.
__global__ void __launch_bounds__(256) compact_kernel(const uint32_t* __restrict__ words, const uint32_t* __restrict__ counts,
                                                      int n_in, int T, long long rows_stride, uint32_t* __restrict__ offs,
                                                      uint16_t* __restrict__ rows) {
  __shared__ uint32_t s_warp[32];
  const int b = blockIdx.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nthr = blockDim.x, nwarps = nthr >> 5;
  const int nwi = (n_in + 31) >> 5;
  const uint32_t* cnt = counts + (size_t)b * T;
  uint32_t* off = offs + (size_t)b * (T + 1);
  const int per = (T + nthr - 1) / nthr;
  const int lo = min(T, tid * per), hi = min(T, lo + per);
  uint32_t sum = 0;
  for (int k = lo; k < hi; ++k) sum += cnt[k];
  uint32_t incl = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const uint32_t x = lane < nwarps ? s_warp[lane] : 0u;
    uint32_t xi = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, xi, o);
      if (lane >= o) xi += y;
    }
    if (lane < nwarps) s_warp[lane] = xi - x;
  }
  __syncthreads();
  uint32_t run = s_warp[warp] + incl - sum;
  for (int k = lo; k < hi; ++k) { off[k] = run; run += cnt[k]; }
  if (lo < hi && hi == T) off[T] = run;
  if (T == 0 && tid == 0) off[0] = 0;
  __syncthreads();
  uint16_t* rw = rows + (size_t)b * rows_stride;
  for (int k = warp; k < T; k += nwarps) {
    uint32_t base = off[k];
    const uint32_t* wk = words + ((size_t)b * T + k) * nwi;
    for (int w0 = 0; w0 < nwi; w0 += 32) {
      const int w = w0 + lane;
      uint32_t word = w < nwi ? wk[w] : 0u;
      if (w == nwi - 1 && (n_in & 31)) word &= (1u << (n_in & 31)) - 1u;
      const int c = __popc(word);
      int inc = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(FULL, inc, o);
        if (lane >= o) inc += y;
      }
      uint32_t pos = base + (uint32_t)(inc - c);
      while (word) {
        const int bp = __ffs(word) - 1;
        word &= word - 1;
        rw[pos++] = (uint16_t)(w * 32 + bp);
      }
      base += (uint32_t)__shfl_sync(FULL, inc, 31);
    }
  }
}

// ====================================================================== main kernel

// S_j over the active rows [r0, r1) of one step: independent loads, unrolled for ILP (eq.(3))
__device__ __forceinline__ int integrate(const uint32_t* __restrict__ wcol, const uint16_t* __restrict__ rows, int r0,
                                        int r1, int wpr, int sh, uint32_t fmask) {
  int S = 0;
  int r = r0;
  for (; r + 4 <= r1; r += 4) {
    const int i0 = rows[r], i1 = rows[r + 1], i2 = rows[r + 2], i3 = rows[r + 3];
    const uint32_t w0 = wcol[i0 * wpr], w1 = wcol[i1 * wpr], w2 = wcol[i2 * wpr], w3 = wcol[i3 * wpr];
    S += (int)(((w0 >> sh) & fmask) + ((w1 >> sh) & fmask) + ((w2 >> sh) & fmask) + ((w3 >> sh) & fmask));
  }
  for (; r < r1; ++r) S += (int)((wcol[(int)rows[r] * wpr] >> sh) & fmask);
  return S;
}

// LTD draws of column j against rows [r0, r0 + n), n <= 32: bit m set iff u_LTD(t, rows[r0+m], j) <= thr.
// Branch-free so that the independent Philox blocks overlap (eq.(7), R13).
__device__ __forceinline__ uint32_t ltd_draws(const uint16_t* __restrict__ rows, int r0, int n, uint32_t t, int j,
                                              uint32_t thr, unsigned long long seed) {
  uint32_t m = 0;
  const int lanej = j & 3;
#pragma unroll 4
  for (int x = 0; x < n; ++x) {
    const uint4 u = philox(t, (uint32_t)rows[r0 + x], (uint32_t)(j >> 2), TAG_LTD, seed);
    m |= (pick(u, lanej) <= thr ? 1u : 0u) << x;
  }
  return m;
}
struct EvLayout {
  size_t slots, wsum, flags, misc, w, pot, dep, dbp, dbd, dtp, dtd, lpre, offs, rows, log, splist, total;
};

__host__ __device__ inline EvLayout ev_layout(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr,
                                              int rows_cap, int offs_cap, int logn) {
  EvLayout L;
  size_t o = 0;
  L.slots = o;  o = align16(o + 2 * kMaxCluster * 2 * 8);   // [parity][rank][2] u64
  L.wsum = o;   o = align16(o + 32 * 2 * 8);                // per warp: summary, key
  L.flags = o;  o = align16(o + 4 * 4);                     // early-stop flag per epoch parity
  L.misc = o;   o = align16(o + 16 * 8);
  L.w = o;      o = align16(o + (size_t)slice_words * 4);
  L.pot = o;    o = align16(o + (size_t)(L_pot > 0 ? L_pot : 1) * 4);
  L.dep = o;    o = align16(o + (size_t)(L_dep > 0 ? L_dep : 1) * 4);
  L.dbp = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.dbd = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.dtp = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.dtd = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.lpre = o;   o = align16(o + (size_t)n_in * 4);
  L.offs = o;   o = align16(o + (size_t)(offs_cap + 1) * 4);
  L.rows = o;   o = align16(o + (size_t)rows_cap * 2);
  L.log = o;    o = align16(o + (size_t)logn * nthr * 4);
  L.splist = o; o = align16(o + (size_t)nthr * 2);
  L.total = o;
  return L;
}

size_t event_smem_bytes(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr, int rows_cap,
                        int offs_cap, int logn) {
  return ev_layout(n_in, slice_words, L_pot, L_dep, q_max, nthr, rows_cap, offs_cap, logn).total;
}

template <bool FIXED>
__global__ void __launch_bounds__(kEvMaxThreads, 1) present_event_kernel(const __grid_constant__ LaunchParams lp) {
  extern __shared__ __align__(16) unsigned char smem[];
  const NetDesc& d0 = lp.descs ? lp.descs[0] : lp.single;
  const int cs = d0.cs;
  const int net = blockIdx.x / cs;
  const int rank = blockIdx.x - net * cs;
  const NetDesc& d = lp.descs ? lp.descs[net] : lp.single;

  const int n_in = d.n_in, n_exc = d.n_exc, bits = d.bits, qmax = d.q_max, wpr = d.wpr, nwe = d.nwe;
  const int T = d.T, flags = d.flags, n_images = d.n_images;
  const int L_pot = d.L_pot, L_dep = d.L_dep, rows_cap = d.rows_cap, offs_cap = d.offs_cap, logn = d.logn;
  const int slice_words = ((n_in * wpr) + 3) & ~3;
  const int nthr = blockDim.x;
  const EvLayout L = ev_layout(n_in, slice_words, L_pot, L_dep, qmax, nthr, rows_cap, offs_cap, logn);
  unsigned long long* s_slots = reinterpret_cast<unsigned long long*>(smem + L.slots);
  unsigned long long* s_wsum = reinterpret_cast<unsigned long long*>(smem + L.wsum);
  int* s_flag = reinterpret_cast<int*>(smem + L.flags);
  int* s_misc = reinterpret_cast<int*>(smem + L.misc);
  uint32_t* s_w = reinterpret_cast<uint32_t*>(smem + L.w);
  uint32_t* s_pot = reinterpret_cast<uint32_t*>(smem + L.pot);
  uint32_t* s_dep = reinterpret_cast<uint32_t*>(smem + L.dep);
  int* s_dbp = reinterpret_cast<int*>(smem + L.dbp);
  int* s_dbd = reinterpret_cast<int*>(smem + L.dbd);
  uint32_t* s_dtp = reinterpret_cast<uint32_t*>(smem + L.dtp);
  uint32_t* s_dtd = reinterpret_cast<uint32_t*>(smem + L.dtd);
  int* s_lpre = reinterpret_cast<int*>(smem + L.lpre);
  uint32_t* s_offs = reinterpret_cast<uint32_t*>(smem + L.offs);
  uint16_t* s_rows = reinterpret_cast<uint16_t*>(smem + L.rows);
  uint32_t* s_log = reinterpret_cast<uint32_t*>(smem + L.log);
  uint16_t* s_splist = reinterpret_cast<uint16_t*>(smem + L.splist);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarps = nthr >> 5;
  const int g0 = (rank * d.ngroups) / cs, g1 = ((rank + 1) * d.ngroups) / cs;
  const int col0 = g0 * 32;
  const int ncols = min(g1 * 32, n_exc) - col0;
  const int ngrp_cta = g1 - g0;
  const bool mycol = tid < ncols;
  const int j = col0 + tid;
  const int lg = bits == 2 ? 4 : (bits == 4 ? 3 : 2);
  const int wj = tid >> lg;
  const int sh = (tid & ((1 << lg) - 1)) * bits;
  const uint32_t fmask = (1u << bits) - 1u;
  const int nq4 = (n_in + 3) >> 2;
  uint32_t* const wcol = s_w + wj;

  Lif lif;
  lif.load(d);
  const bool fixed = lif.fixed;
  const int vreset = fixed ? d.Vreset : __float_as_int(d.vresetf);
  const int vinit = fixed ? d.Vinit : __float_as_int(d.vinitf);
  const int t_ref = d.t_ref, t_inh = d.t_inh, t_ltp = d.t_ltp;
  const bool hard = d.wta_mode == 0;
  const bool stoch = d.stdp_mode == 0;
  const bool inh_reset = d.inh_mode == 0;
  const bool keep = (flags & FLAG_KEEP_STATE) != 0;
  const int tbase = keep ? d.t0 : 0;

  // ---- one-time staging
  for (int k = tid; k < L_pot; k += nthr) s_pot[k] = d.pot_m1[k];
  for (int k = tid; k < L_dep; k += nthr) s_dep[k] = d.dep_m1[k];
  for (int k = tid; k <= qmax; k += nthr) {
    s_dbp[k] = d.det_base_p[k]; s_dbd[k] = d.det_base_d[k];
    s_dtp[k] = d.det_thr_p[k];  s_dtd[k] = d.det_thr_d[k];
  }
  {
    const uint4* src = reinterpret_cast<const uint4*>(d.wslices + (size_t)rank * slice_words);
    uint4* dst = reinterpret_cast<uint4*>(s_w);
    for (int k = tid; k < slice_words / 4; k += nthr) dst[k] = src[k];
  }
  if (tid == 0) { s_flag[0] = INT_MAX; s_flag[1] = INT_MAX; }
  int v = vinit, cnt = 0, lpost = kNever;
  if (keep) {
    if (mycol) { v = d.v[j]; cnt = d.cnt[j]; lpost = d.last_post[j]; }
    for (int i = tid; i < n_in; i += nthr) s_lpre[i] = d.last_pre[i];
  }
  uint32_t ltd_trials = 0, ltd_events = 0, ltp_trials = 0, ltp_events = 0;   // per launch, < 2^32
  unsigned long long act_sum = 0, post_sum = 0;
  uint32_t eng_epochs = 0, eng_hz = 0, eng_resim = 0, eng_spec = 0, eng_undo = 0;
  // every CTA of the cluster has initialised its flags before any remote red.min can target them
  if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }

  int ep = 0;
  unsigned long long* trace = d.trace ? d.trace + (size_t)rank * d.trace_cap * 8 : nullptr;
  unsigned long long* s_tmax = reinterpret_cast<unsigned long long*>(s_misc + 8);   // max speculation end
  unsigned long long tr0 = 0, tr2 = 0, tr3 = 0;
  for (int b = 0; b < n_images; ++b) {
    const unsigned long long seed = d.seeds[b];
    if (!keep) {
      v = vinit; cnt = 0; lpost = kNever;
      for (int i = tid; i < n_in; i += nthr) s_lpre[i] = kNever;
    }
    const uint32_t* offs_g = d.ev_offs + (size_t)b * (T + 1);
    const uint16_t* rows_g = d.ev_rows + (size_t)b * d.rows_stride;
    const bool last_img = (b == n_images - 1);
    const bool rec_out = last_img && d.raster_out != nullptr;
    int img_spikes = 0;
    int ka = 0, kb = 0;
    uint32_t wbase = 0;
    int k0 = 0;
    if (rank == 0 && tid == 0 && T > 0) act_sum += (unsigned long long)(offs_g[T] - offs_g[0]);
    __syncthreads();

    while (k0 < T) {
      // ---------------------------------------------------------- stage the active-row window
      if (k0 >= kb) {
        ka = k0;
        const int n_o = min(offs_cap, T - ka);
        for (int x = tid; x <= n_o; x += nthr) s_offs[x] = offs_g[ka + x];
        if (tid == 0) s_misc[0] = 0;
        __syncthreads();
        wbase = s_offs[0];
        int fit = 0;
        for (int x = tid + 1; x <= n_o; x += nthr) fit += (s_offs[x] - wbase <= (uint32_t)rows_cap) ? 1 : 0;
        if (fit) atomicAdd(&s_misc[0], fit);
        __syncthreads();
        const int nsteps = s_misc[0];          // >= 1: rows_cap >= n_in
        kb = ka + nsteps;
        const uint32_t nrows = s_offs[nsteps] - wbase;
        for (uint32_t x = tid; x < nrows; x += nthr) s_rows[x] = rows_g[wbase + x];
        __syncthreads();
      }
      const int kend = kb;
      const int fp = ep & 1;
      if (trace && tid == 0) { tr0 = globaltimer(); *s_tmax = 0ull; }

      // ---------------------------------------------------------- speculation (column-local, no barriers)
      int p = kend;            // first step not fully processed by this thread
      bool cand = false;       // stopped at its own threshold crossing at p (LIF done, LTD pending)
      bool hz = false;         // stopped at p with nothing done (undo log full)
      const int v0 = v, cnt0 = cnt;
      int v1 = v, cnt1 = cnt, vb = v;
      int nlog = 0;
      {
        // Warp-synchronous speculation: every lane of the warp walks the same step kk (lanes that
        // stopped are predicated off), so the LTD Philox blocks of an LTD-active column can be
        // spread over all 32 lanes (one block per row) instead of serialised in one lane.
        const uint32_t flag_addr = smem_u32(&s_flag[fp]);
        const bool ltd_col = mycol && stoch && lpost >= 0;
        const int jw = col0 + warp * 32;                          // column of lane 0 of this warp
        bool done = !mycol;
        int kk = k0;
        int r0 = (int)(s_offs[k0 - ka] - wbase);
        auto signal = [&](int f) {                                // tell the cluster where to stop
          atomicMin(&s_flag[fp], f);
          for (int r = 0; r < cs; ++r)
            if (r != rank) red_min_cluster(&s_flag[fp], (uint32_t)r, f);
        };
        while (__any_sync(FULL, !done)) {
          if (!done && (kk >= kend || kk > ld_volatile_shared_u32addr(flag_addr))) { done = true; p = kk; }
          if (kk >= kend) break;                                  // warp-uniform
          const int r1 = (int)(s_offs[kk - ka + 1] - wbase);
          const int t = tbase + kk;
          bool ltd_on = false;
          int cb = cnt;
          if (!done) {
            const int S = integrate(wcol, s_rows, r0, r1, wpr, sh, fmask);   // (a2) eq.(3)
            if (cnt > 0) {
              --cnt;                                               // (a3) refractory / inhibited: hold v
            } else {
              vb = v;
              if (lif.step_t<FIXED>(v, S)) { cand = true; done = true; p = kk; signal(kk); }   // (a3) eqs.(1)(2)
            }
            ltd_on = !done && ltd_col && (t - lpost) < L_dep;
          }
          // (a5) LTD, eq.(7), exact (R10, R14): cooperative draws, then this lane's events
          const uint32_t lmask = __ballot_sync(FULL, ltd_on);
          if (lmask) {
            const uint32_t thr = ltd_on ? s_dep[t - lpost] : 0u;
            const int nlog_step = nlog;
            bool overflow = false;
            uint32_t ev_step = 0;
            for (int c0 = r0; c0 < r1; c0 += 32) {               // warp-uniform chunks of <= 32 rows
              const int n = min(32, r1 - c0);
              const uint32_t row_here = lane < n ? (uint32_t)s_rows[c0 + lane] : 0u;
              uint32_t mine = 0;
              for (uint32_t lm = lmask; lm; lm &= lm - 1) {
                const int L = __ffs(lm) - 1;
                const int jL = jw + L;
                const uint32_t thrL = __shfl_sync(FULL, thr, L);
                bool bit = false;
                if (lane < n) {
                  const uint4 u = philox((uint32_t)t, row_here, (uint32_t)(jL >> 2), TAG_LTD, seed);
                  bit = pick(u, jL & 3) <= thrL;
                }
                const uint32_t m = __ballot_sync(FULL, bit);
                if (lane == L) mine = m;
              }
              if (ltd_on && !overflow) {
                while (mine) {
                  const int x = __ffs(mine) - 1;
                  mine &= mine - 1;
                  if (kk > k0 && nlog == logn) { overflow = true; break; }
                  const int i = s_rows[c0 + x];
                  uint32_t* pw = wcol + i * wpr;
                  const bool applied = ((*pw >> sh) & fmask) != 0u;
                  if (applied) atomicSub(pw, 1u << sh);
                  ++ev_step;
                  if (kk > k0)
                    s_log[nlog++ * nthr + tid] = ((uint32_t)(kk - k0) << 16) | (applied ? 0x8000u : 0u) | (uint32_t)i;
                }
              }
            }
            if (ltd_on) {
              if (overflow) {                                      // undo this step entirely; stop before it
                while (nlog > nlog_step) {
                  const uint32_t e = s_log[(nlog - 1) * nthr + tid];
                  if (e & 0x8000u) atomicAdd(wcol + (int)(e & 0x7FFFu) * wpr, 1u << sh);
                  --nlog;
                }
                cnt = cb;
                if (cb == 0) v = vb;
                hz = true;
                done = true;
                p = kk;
                ++eng_hz;
                signal(kk - 1);
              } else {
                ltd_events += ev_step;
                ltd_trials += (uint32_t)(r1 - r0);
              }
            }
          }
          if (!done && kk == k0) { v1 = v; cnt1 = cnt; }
          ++kk;
          r0 = r1;
        }
        if (!mycol) p = kend;
        if (mycol) eng_spec += (uint32_t)(p - k0 + (cand ? 1 : 0));
      }

      if (trace && lane == 0) atomicMax(s_tmax, globaltimer());
      // ---------------------------------------------------------- CTA summary -> cluster exchange
      {
        const uint32_t w1 = ((uint32_t)(0xFFFF - min(p, kend)) << 1) | (hz ? 1u : 0u);
        const uint32_t W1w = __reduce_max_sync(FULL, w1);
        const int Pw = 0xFFFF - (int)(W1w >> 1);
        const bool c_at = cand && p == Pw;
        const uint32_t kh = c_at ? lif.ord(v) : 0u;
        const uint32_t mh = __reduce_max_sync(FULL, kh);
        const uint32_t ml = __reduce_max_sync(FULL, (c_at && kh == mh) ? (0xFFFFFFFFu - (uint32_t)j) : 0u);
        const uint32_t cw = (uint32_t)__popc(__ballot_sync(FULL, c_at));
        if (lane == 0) {
          s_wsum[2 * warp] = ((unsigned long long)W1w << 32) | cw;
          s_wsum[2 * warp + 1] = ((unsigned long long)mh << 32) | ml;
        }
      }
      __syncthreads();                                                               // S1
      if (trace && tid == 0) tr2 = globaltimer();
      if (warp == 0) {
        const unsigned long long a = lane < nwarps ? s_wsum[2 * lane] : 0ull;
        const unsigned long long k = lane < nwarps ? s_wsum[2 * lane + 1] : 0ull;
        const uint32_t W1c = __reduce_max_sync(FULL, (uint32_t)(a >> 32));
        const bool at = lane < nwarps && (uint32_t)(a >> 32) == W1c;
        const uint32_t cc = __reduce_add_sync(FULL, at ? (uint32_t)a : 0u);
        const uint32_t kh = __reduce_max_sync(FULL, at ? (uint32_t)(k >> 32) : 0u);
        const uint32_t kl = __reduce_max_sync(FULL, (at && (uint32_t)(k >> 32) == kh) ? (uint32_t)k : 0u);
        const unsigned long long A = ((unsigned long long)W1c << 32) | cc;
        const unsigned long long K = ((unsigned long long)kh << 32) | kl;
        unsigned long long* slot = s_slots + (size_t)(fp * kMaxCluster + rank) * 2;
        if (cs == 1) {
          if (lane == 0) { slot[0] = A; slot[1] = K; }
        } else if (lane < cs) {
          st_cluster_u64(slot, (uint32_t)lane, A);
          st_cluster_u64(slot + 1, (uint32_t)lane, K);
        }
        if (lane == 0) { s_flag[fp ^ 1] = INT_MAX; s_misc[1] = 0; }
      }
      if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }   // the one cross-SM exchange
      if (trace && tid == 0) tr3 = globaltimer();

      // ---------------------------------------------------------- global decision
      uint32_t W1 = 0, count = 0;
      unsigned long long K = 0;
      for (int r = 0; r < cs; ++r) W1 = max(W1, (uint32_t)(s_slots[(size_t)(fp * kMaxCluster + r) * 2] >> 32));
      for (int r = 0; r < cs; ++r) {
        const unsigned long long A = s_slots[(size_t)(fp * kMaxCluster + r) * 2];
        if ((uint32_t)(A >> 32) == W1) {
          count += (uint32_t)A;
          const unsigned long long kk = s_slots[(size_t)(fp * kMaxCluster + r) * 2 + 1];
          K = kk > K ? kk : K;
        }
      }
      const int P = 0xFFFF - (int)(W1 >> 1);
      const bool unknown = (W1 & 1u) != 0u;
      const bool at_end = P >= kend;
      const bool event = !at_end && !unknown;
      const int tP = tbase + P;

      // ---------------------------------------------------------- per-thread resolution / rollback
      // resim(X): state after step k0 + undo of every logged LTD, then replay k0+1..X exactly.
      auto count_trials = [&](int from, int to) -> uint32_t {   // LTD trials of steps [from, to)
        uint32_t n = 0;
        if (stoch && lpost >= 0)
          for (int kk = from; kk < to; ++kk)
            if ((tbase + kk - lpost) < L_dep) n += s_offs[kk - ka + 1] - s_offs[kk - ka];
        return n;
      };
      auto undo_after = [&](int rel_keep) {       // undo logged LTD of steps k0+rel > k0+rel_keep
        while (nlog > 0) {
          const uint32_t e = s_log[(nlog - 1) * nthr + tid];
          if ((int)(e >> 16) <= rel_keep) break;
          if (e & 0x8000u) atomicAdd(wcol + (int)(e & 0x7FFFu) * wpr, 1u << sh);
          --ltd_events;
          --nlog;
          ++eng_undo;
        }
      };
      auto resim = [&](int X) {
        ++eng_resim;
        undo_after(0);
        ltd_trials -= count_trials(k0 + 1, p);
        v = v1; cnt = cnt1;
        for (int kk = k0 + 1; kk <= X; ++kk) {
          const int r0 = (int)(s_offs[kk - ka] - wbase), r1 = (int)(s_offs[kk - ka + 1] - wbase);
          const int t = tbase + kk;
          const int S = integrate(wcol, s_rows, r0, r1, wpr, sh, fmask);
          if (cnt > 0) --cnt; else lif.step_t<FIXED>(v, S);
          if (stoch && lpost >= 0 && (t - lpost) < L_dep) {
            const uint32_t thr = s_dep[t - lpost];
            for (int c0 = r0; c0 < r1; c0 += 32) {
              uint32_t m = ltd_draws(s_rows, c0, min(32, r1 - c0), (uint32_t)t, j, thr, seed);
              while (m) {
                const int x = __ffs(m) - 1;
                m &= m - 1;
                uint32_t* pw = wcol + (int)s_rows[c0 + x] * wpr;
                if ((*pw >> sh) & fmask) atomicSub(pw, 1u << sh);
                ++ltd_events;
              }
            }
            ltd_trials += (uint32_t)(r1 - r0);
          }
        }
      };
      if (mycol && !at_end) {
        if (event) {
          if (p > P) {                                   // ran past t*: rebuild the state after step t*
            if (inh_reset) {
              undo_after(P - k0);
              ltd_trials -= count_trials(P + 1, p);
              cnt = max(cnt0 - (P - k0 + 1), 0);        // no crossing in [k0, t*]: cnt only counted down
              (void)v0;
            } else {
              resim(P);
            }
          }
        } else {                                         // unknown at P: commit only through P - 1
          if (p == P) {
            if (cand) v = vb;
          } else {
            resim(P - 1);
          }
        }
      }
      bool spiked = false;
      uint32_t W = 0xFFFFFFFFu;
      if (event) {
        if (hard) {
          W = 0xFFFFFFFFu - (uint32_t)K;
          if (mycol) {
            if ((uint32_t)j == W) { v = vreset; cnt = t_ref; spiked = true; }
            else { cnt = max(cnt, t_inh); if (inh_reset) v = vreset; }
          }
          img_spikes += 1;
        } else {
          if (mycol) {
            const bool me = cand && p == P;
            if (me) { v = vreset; cnt = t_ref; spiked = true; }
            if (count >= 2u || !me) { cnt = max(cnt, t_inh); if (inh_reset) v = vreset; }
          }
          img_spikes += (int)count;
        }
        // pending LTD at t* of the columns that stopped there (old last_post, R14)
        if (mycol && cand && p == P && stoch && lpost >= 0 && (tP - lpost) < L_dep) {
          const int r0 = (int)(s_offs[P - ka] - wbase), r1 = (int)(s_offs[P - ka + 1] - wbase);
          const uint32_t thr = s_dep[tP - lpost];
          for (int c0 = r0; c0 < r1; c0 += 32) {
            uint32_t m = ltd_draws(s_rows, c0, min(32, r1 - c0), (uint32_t)tP, j, thr, seed);
            while (m) {
              const int x = __ffs(m) - 1;
              m &= m - 1;
              uint32_t* pw = wcol + (int)s_rows[c0 + x] * wpr;
              if ((*pw >> sh) & fmask) atomicSub(pw, 1u << sh);
              ++ltd_events;
            }
          }
          ltd_trials += (uint32_t)(r1 - r0);
        }
        if (rec_out) {
          const uint32_t bal = __ballot_sync(FULL, spiked);
          if (lane == 0 && warp < ngrp_cta) d.raster_out[(size_t)P * nwe + g0 + warp] = bal;
        }
        if (spiked && !hard) { const int pos = atomicAdd(&s_misc[1], 1); s_splist[pos] = (uint16_t)tid; }
      }
      const int k_last = event ? P : (at_end ? kend - 1 : P - 1);
      __syncthreads();                                                               // S2
      // spike timers of the inputs through the committed step
      for (int kk = k0 + tid; kk <= k_last; kk += nthr) {
        const int r0 = (int)(s_offs[kk - ka] - wbase), r1 = (int)(s_offs[kk - ka + 1] - wbase);
        for (int r = r0; r < r1; ++r) atomicMax(&s_lpre[s_rows[r]], tbase + kk);
      }
      const bool local_spike = event && (hard ? (W >= (uint32_t)col0 && W < (uint32_t)(col0 + ncols)) : false);
      __syncthreads();                                                               // S3
      if (trace && tid == 0 && ep < d.trace_cap) trace[(size_t)ep * 8 + 6] = globaltimer();
      const int nsp = hard ? (local_spike ? 1 : 0) : (event ? s_misc[1] : 0);
      if (nsp > 0) {
        // (a5) LTP eq.(6) / (a6) deterministic arm at t*, rows spread over threads (row words owned)
        for (int grp = tid; grp < nq4; grp += nthr) {
          for (int m = 0; m < nsp; ++m) {
            const int Wl = hard ? (int)(W - (uint32_t)col0) : (int)s_splist[m];
            const int Wg = col0 + Wl;
            const int ww = Wl >> lg, wsh = (Wl & ((1 << lg) - 1)) * bits;
            const uint4 u = philox((uint32_t)tP, (uint32_t)Wg, (uint32_t)grp, stoch ? TAG_LTP : TAG_ROUND, seed);
#pragma unroll
            for (int r = 0; r < 4; ++r) {
              const int i = 4 * grp + r;
              if (i >= n_in) break;
              const int lpi = s_lpre[i];
              uint32_t* pw = s_w + i * wpr + ww;
              if (stoch) {
                if (lpi < 0) continue;
                const int D = tP - lpi;
                if (D >= L_pot) continue;
                ++ltp_trials;
                if (pick(u, r) <= s_pot[D]) {
                  ++ltp_events;
                  const uint32_t word = *pw;
                  if (((word >> wsh) & fmask) < (uint32_t)qmax) *pw = word + (1u << wsh);
                }
              } else {
                const uint32_t word = *pw;
                const int q0 = (int)((word >> wsh) & fmask);
                const bool pot = lpi >= 0 && (tP - lpi) <= t_ltp;
                const int base = pot ? s_dbp[q0] : s_dbd[q0];
                const uint32_t thr = pot ? s_dtp[q0] : s_dtd[q0];
                const int dq = base + (pick(u, r) < thr ? 1 : 0);
                int q1 = pot ? q0 + dq : q0 - dq;
                q1 = q1 < 0 ? 0 : (q1 > qmax ? qmax : q1);
                *pw = (word & ~(fmask << wsh)) | ((uint32_t)q1 << wsh);
                if (pot) { ++ltp_trials; if (dq > 0) ++ltp_events; }
                else     { ++ltd_trials; if (dq > 0) ++ltd_events; }
              }
            }
          }
        }
        __syncthreads();                                                             // S4
      }
      if (spiked) lpost = tP;
      if (trace && tid == 0 && ep < d.trace_cap) {
        unsigned long long* rec = trace + (size_t)ep * 8;
        rec[0] = ((unsigned long long)b << 32) | (unsigned)k0;
        rec[1] = ((unsigned long long)(event ? 1 : (unknown ? 2 : 0)) << 32) | (unsigned)P;
        rec[2] = tr0; rec[3] = *s_tmax; rec[4] = tr2; rec[5] = tr3; rec[7] = globaltimer();
      }
      k0 = k_last + 1;
      ++ep;
      ++eng_epochs;
    }  // epochs

    if (rank == 0 && tid == 0) {
      post_sum += (unsigned long long)img_spikes;
      if (d.spike_counts) d.spike_counts[b] = img_spikes;
    }
    if (last_img) {
      if (mycol) { d.v[j] = v; d.cnt[j] = cnt; d.last_post[j] = lpost; }
      if (rank == 0) for (int i = tid; i < n_in; i += nthr) d.last_pre[i] = s_lpre[i];
    }
    __syncthreads();
  }  // images

  {
    uint4* dst = reinterpret_cast<uint4*>(d.wslices + (size_t)rank * slice_words);
    const uint4* src = reinterpret_cast<const uint4*>(s_w);
    for (int k = tid; k < slice_words / 4; k += nthr) dst[k] = src[k];
  }
  {
    unsigned long long a = ltd_trials, b2 = ltd_events, c = ltp_trials, e = ltp_events;  // widen before the warp sum
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
      atomicAdd(&d.stats[6], (unsigned long long)n_images);
      atomicAdd(&d.stats[7], (unsigned long long)n_images * (unsigned long long)T);
      atomicAdd(&d.stats[8], (unsigned long long)eng_epochs);
    }
    unsigned long long h2 = eng_hz, r2 = eng_resim, s2 = eng_spec, u2 = eng_undo;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      h2 += __shfl_xor_sync(FULL, h2, o); r2 += __shfl_xor_sync(FULL, r2, o);
      s2 += __shfl_xor_sync(FULL, s2, o); u2 += __shfl_xor_sync(FULL, u2, o);
    }
    if (lane == 0) {
      if (h2) atomicAdd(&d.stats[9], h2);
      if (r2) atomicAdd(&d.stats[10], r2);
      if (s2) atomicAdd(&d.stats[11], s2);
      if (u2) atomicAdd(&d.stats[12], u2);
    }
  }
  if (cs > 1) { cluster_arrive(); cluster_wait(); }
}

// ====================================================================== host launchers
static unsigned cdiv(long long a, long long b) { return (unsigned)((a + b - 1) / b); }

cudaError_t launch_encode(const uint8_t* images, const unsigned long long* thr_enc, const unsigned long long* seeds,
                          int n_in, int T, int n_images, int t0, uint32_t* words, uint32_t* counts, cudaStream_t s) {
  if (T <= 0 || n_images <= 0) return cudaSuccess;
  dim3 grid(cdiv(T, kEncWarps), (unsigned)n_images);
  encode_kernel<<<grid, kEncWarps * 32, 0, s>>>(images, thr_enc, seeds, n_in, T, t0, words, counts);
  return cudaGetLastError();
}

cudaError_t launch_counts_from_raster(const uint32_t* raster, int n_in, int T, uint32_t* counts, cudaStream_t s) {
  if (T <= 0) return cudaSuccess;
  counts_from_raster_kernel<<<cdiv(T, 4), 128, 0, s>>>(raster, n_in, T, counts);
  return cudaGetLastError();
}

cudaError_t launch_compact(const uint32_t* words, const uint32_t* counts, int n_in, int T, int n_images,
                           long long rows_stride, uint32_t* offs, uint16_t* rows, cudaStream_t s) {
  if (n_images <= 0) return cudaSuccess;
  compact_kernel<<<(unsigned)n_images, 256, 0, s>>>(words, counts, n_in, T, rows_stride, offs, rows);
  return cudaGetLastError();
}

template <bool FIXED>
static cudaError_t configure_event(size_t smem, int cs) {
  cudaError_t e = cudaFuncSetAttribute(present_event_kernel<FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (cs > 8) e = cudaFuncSetAttribute(present_event_kernel<FIXED>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  return e;
}

static void fill_cfg_ev(cudaLaunchConfig_t& cfg, cudaLaunchAttribute* attr, int n_nets, int cs, int nthr, size_t smem,
                        cudaStream_t s) {
  cfg = cudaLaunchConfig_t{};
  cfg.gridDim = dim3((unsigned)(n_nets * cs));
  cfg.blockDim = dim3((unsigned)nthr);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.attrs = attr;
  cfg.numAttrs = 0;
  if (cs > 1) {
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.numAttrs = 1;
  }
}

cudaError_t query_max_clusters_event(int cs, int nthr, size_t smem, int* out) {
  cudaError_t e = configure_event<false>(smem, cs);
  if (e == cudaSuccess) e = configure_event<true>(smem, cs);
  if (e != cudaSuccess) return e;
  if (cs == 1) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(out, present_event_kernel<false>, nthr, smem);
  cudaLaunchConfig_t cfg;
  cudaLaunchAttribute attr[1];
  fill_cfg_ev(cfg, attr, 1, cs, nthr, smem, 0);
  return cudaOccupancyMaxActiveClusters(out, present_event_kernel<false>, &cfg);
}

cudaError_t launch_present_event(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, cudaStream_t s) {
  const bool fixed = (lp.descs ? 0 : lp.single.membrane_mode) == 1;   // ensembles: see launch_present_event_mode
  cudaError_t e = fixed ? configure_event<true>(smem, cs) : configure_event<false>(smem, cs);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg;
  cudaLaunchAttribute attr[1];
  fill_cfg_ev(cfg, attr, n_nets, cs, nthr, smem, s);
  return fixed ? cudaLaunchKernelEx(&cfg, present_event_kernel<true>, lp)
               : cudaLaunchKernelEx(&cfg, present_event_kernel<false>, lp);
}

cudaError_t launch_present_event_mode(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, int fixed,
                                      cudaStream_t s) {
  cudaError_t e = fixed ? configure_event<true>(smem, cs) : configure_event<false>(smem, cs);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg;
  cudaLaunchAttribute attr[1];
  fill_cfg_ev(cfg, attr, n_nets, cs, nthr, smem, s);
  return fixed ? cudaLaunchKernelEx(&cfg, present_event_kernel<true>, lp)
               : cudaLaunchKernelEx(&cfg, present_event_kernel<false>, lp);
}

}  // namespace snn
