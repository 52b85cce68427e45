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

// ablation switch for timing experiments only (tools/ablate.sh); 0 in every shipped build
#ifndef SNN_EXP
#define SNN_EXP 0
#endif

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
                                                      uint16_t* __restrict__ rows, uint16_t* __restrict__ rows16) {
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
    const uint32_t kbase = base;
    uint16_t* r16 = rows16 + ((size_t)b * T + k) * kPadRows;
    if (lane < kPadRows) r16[lane] = (uint16_t)n_in;          // padding -> the all-zero weight row
    __syncwarp();
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
        if (pos - kbase < (uint32_t)kPadRows) r16[pos - kbase] = (uint16_t)(w * 32 + bp);
        rw[pos++] = (uint16_t)(w * 32 + bp);
      }
      base += (uint32_t)__shfl_sync(FULL, inc, 31);
    }
  }
}

// ====================================================================== main kernel
// Thread -> column mapping: the slice is packed row-major, word w of a row holds
// local columns w*cpw .. w*cpw+cpw-1 (cpw = 32/BITS).  Four threads share a word: thread
// (w, f) owns the CPT = 8/BITS columns at fields f, f+4, f+8, f+12, which sit LW = 32/CPT bits
// apart, so one shift+mask of the word yields all of the thread's codes in separate SWAR lanes
// and one add integrates all of them (eq.(3)).
constexpr int kBlk = 8;             // steps per speculation block

// Swar<BITS, CPT>: a thread owns CPT columns of one packed word, LW = 32/CPT bits apart; TPW = CPW/CPT
// threads share the word.  One shift+mask yields the thread's CPT codes in separate SWAR lanes.
template <int BITS, int CPT_> struct Swar {
  static constexpr int CPT = CPT_;
  static constexpr int CPW = 32 / BITS;
  static constexpr int TPW = CPW / CPT_;
  static constexpr int LW = 32 / CPT_;
  static constexpr uint32_t FM = (1u << BITS) - 1u;
  static constexpr uint32_t LMASK = CPT_ == 1 ? FM : (CPT_ == 2 ? (FM | (FM << 16)) : (FM * 0x01010101u));
  // rows that can be summed before a lane overflows
  static constexpr int CHUNK = CPT_ == 1 ? (1 << 30) : (int)(((1u << (LW & 31)) - 1u) / FM);
};
// S[c] = sum over the active rows [r0, r1) of the thread's CPT codes (exact; lanes never overflow)
template <int BITS, int CPT_>
__device__ __forceinline__ void integrate_swar(const uint32_t* __restrict__ wcol, const uint16_t* __restrict__ rows,
                                               int r0, int r1, int wpr, int fsh, int (&S)[CPT_]) {
  using Z = Swar<BITS, CPT_>;
#pragma unroll
  for (int c = 0; c < Z::CPT; ++c) S[c] = 0;
  int r = r0;
  while (r < r1) {
    const int rend = min(r1, r + Z::CHUNK);
    uint32_t acc = 0;
    for (; r + 4 <= rend; r += 4) {
      const int i0 = rows[r], i1 = rows[r + 1], i2 = rows[r + 2], i3 = rows[r + 3];
      const uint32_t w0 = wcol[i0 * wpr], w1 = wcol[i1 * wpr], w2 = wcol[i2 * wpr], w3 = wcol[i3 * wpr];
      acc += ((w0 >> fsh) & Z::LMASK) + ((w1 >> fsh) & Z::LMASK) + ((w2 >> fsh) & Z::LMASK) + ((w3 >> fsh) & Z::LMASK);
    }
    for (; r < rend; ++r) acc += (wcol[(int)rows[r] * wpr] >> fsh) & Z::LMASK;
#pragma unroll
    for (int c = 0; c < Z::CPT; ++c)
      S[c] += (int)(Z::LW == 32 ? acc : ((acc >> (c * Z::LW)) & ((1u << (Z::LW & 31)) - 1u)));
  }
}

// lane-wise max of two SWAR words (lanes of 32/CPT bits)
template <int CPT>
__device__ __forceinline__ uint32_t vmax_lanes(uint32_t a, uint32_t b) {
  if constexpr (CPT == 4) return __vmaxu4(a, b);
  else if constexpr (CPT == 2) return __vmaxu2(a, b);
  else return a > b ? a : b;
}


// Window row metadata (one u32 per active row): word offset row*wpr (bits 0..15; the slice holds
// < 2^16 words), step within the window (bits 16..24), distance to the next occurrence of the same
// input within the next 64 rows (bits 25..31, 0 = none).
__device__ __forceinline__ uint32_t meta_woff(uint32_t m) { return m & 0xFFFFu; }
__device__ __forceinline__ int meta_step(uint32_t m) { return (int)((m >> 16) & 0x1FFu); }
__device__ __forceinline__ uint32_t meta_link(uint32_t m) { return m >> 25; }

// LTD decrement of the row at window position r (step b of the block): the later block steps that
// contain the same input were summed with the old code, so every later occurrence q (followed through
// the next-occurrence links) lowers the running sums of every non-empty block step >= step(q) by
// delta (the LIF chain reads only the slots of non-empty steps).
__device__ __forceinline__ void block_correct(const uint32_t* __restrict__ meta, uint32_t* my_acc, int nthr, int r,
                                              int rblk1, int sbase, uint32_t nonempty, uint32_t delta) {
  uint32_t lk = meta_link(meta[r]);
  int q = r + (int)lk;
  while (lk != 0u && q < rblk1) {
    const uint32_t rs = meta[q];
    const int s2 = meta_step(rs) - sbase;
#pragma unroll 1
    for (uint32_t m = nonempty & (0xFFFFFFFFu << s2); m; m &= m - 1u) my_acc[(__ffs(m) - 1) * nthr] += delta;
    lk = meta_link(rs);
    q += (int)lk;
  }
}

struct EvLayout {
  size_t slots, wsum, flags, misc, w, pot, dep, dbp, dbd, dtp, dtd, lpre, lpost, offs, binfo, rows, meta, ev, acc, log, total;
};

__host__ __device__ inline EvLayout ev_layout(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr,
                                              int rows_cap, int offs_cap, int logn) {
  EvLayout L;
  size_t o = 0;
  L.slots = o;  o = align16(o + 2 * kMaxCluster * 2 * 8);   // [parity][rank][2] u64
  L.wsum = o;   o = align16(o + 32 * 2 * 8);                // per warp: summary, key
  L.flags = o;  o = align16(o + 4 * 4);                     // early-stop flag per epoch parity
  L.misc = o;   o = align16(o + 16 * 8 + (size_t)nthr * 4 * 4 + 16 + 32 * 16);   // header, spikers, warp prof
  L.w = o;      o = align16(o + (size_t)slice_words * 4);
  L.pot = o;    o = align16(o + (size_t)(L_pot > 0 ? L_pot : 1) * 4);
  L.dep = o;    o = align16(o + (size_t)(L_dep > 0 ? L_dep : 1) * 4);
  L.dbp = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.dbd = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.dtp = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.dtd = o;    o = align16(o + (size_t)(q_max + 1) * 4);
  L.lpre = o;   o = align16(o + (size_t)n_in * 4);
  L.lpost = o;  o = align16(o + (size_t)nthr * 4 * 4);        // last_post of the CTA's local columns
  L.offs = o;   o = align16(o + (size_t)(offs_cap + 1) * 4);
  L.binfo = o;  o = align16(o + (size_t)offs_cap * 4);               // block shape from every window step
  L.rows = o;   o = align16(o + (size_t)(rows_cap + 2) * 2);         // input id of every window row (+ pad)
  L.meta = o;   o = align16(o + (size_t)(rows_cap + 8) * 4);         // row metadata (+ 8 zero-row pads)
  L.ev = o;     o = align16(o + (size_t)8 * nthr * 4);               // block LTD event masks [c][2][thread]
  L.acc = o;    o = align16(o + (size_t)(kBlk + 1) * nthr * 4);      // block SWAR sums [b][thread] + spill slot
  L.log = o;    o = align16(o + (size_t)logn * nthr * 4);
  L.total = o;
  return L;
}

size_t event_smem_bytes(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr, int rows_cap,
                        int offs_cap, int logn) {
  return ev_layout(n_in, slice_words, L_pot, L_dep, q_max, nthr, rows_cap, offs_cap, logn).total;
}

// undo-log entry: rel step (16) | column slot c (2) | applied (1) | row (13)
__device__ __forceinline__ uint32_t log_entry(int rel, int c, bool applied, int row) {
  return ((uint32_t)rel << 16) | ((uint32_t)c << 14) | (applied ? 0x2000u : 0u) | (uint32_t)row;
}

template <int BITS, int CPT_, bool FIXED>
__global__ void __launch_bounds__(kEvMaxThreads, 1) present_event_kernel(const __grid_constant__ LaunchParams lp) {
  using Z = Swar<BITS, CPT_>;
  constexpr int CPT = Z::CPT;
  constexpr int CPW = Z::CPW;
  constexpr int TPW = Z::TPW;
  constexpr uint32_t FMASK = (1u << BITS) - 1u;
  extern __shared__ __align__(16) unsigned char smem[];
  const NetDesc& d0 = lp.descs ? lp.descs[0] : lp.single;
  const int cs = d0.cs;
  const int net = blockIdx.x / cs;
  const int rank = blockIdx.x - net * cs;
  const NetDesc& d = lp.descs ? lp.descs[net] : lp.single;

  const int n_in = d.n_in, n_exc = d.n_exc, qmax = d.q_max, wpr = d.wpr, nwe = d.nwe;
  const int T = d.T, flags = d.flags, n_images = d.n_images;
  const int L_pot = d.L_pot, L_dep = d.L_dep, rows_cap = d.rows_cap, offs_cap = d.offs_cap, logn = d.logn;
  const int slice_words = d.slice_words;
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
  int* s_lpost = reinterpret_cast<int*>(smem + L.lpost);
  uint32_t* s_offs = reinterpret_cast<uint32_t*>(smem + L.offs);
  uint32_t* s_binfo = reinterpret_cast<uint32_t*>(smem + L.binfo);
  uint16_t* s_rows = reinterpret_cast<uint16_t*>(smem + L.rows);
  uint32_t* s_meta = reinterpret_cast<uint32_t*>(smem + L.meta);
  uint32_t* s_ev = reinterpret_cast<uint32_t*>(smem + L.ev);
  uint32_t* s_acc = reinterpret_cast<uint32_t*>(smem + L.acc);
  uint32_t* s_log = reinterpret_cast<uint32_t*>(smem + L.log);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarps = nthr >> 5;
  const int g0 = (rank * d.ngroups) / cs, g1 = ((rank + 1) * d.ngroups) / cs;
  const int col0 = g0 * 32;
  const int cbase = d.col_base;                              // global index of local column 0 (shards)
  const int ncols = min(g1 * 32, n_exc) - col0;
  // this thread's word and columns
  const int wj = tid / TPW, f = tid % TPW;
  const int fsh = f * BITS;                                  // SWAR shift of the thread's lanes
  uint32_t* const wcol = s_w + wj;
  int jcol[CPT];                                             // global column of slot c (or -1)
  uint32_t valid = 0;
#pragma unroll
  for (int c = 0; c < CPT; ++c) {
    const int jl = wj * CPW + f + TPW * c;
    jcol[c] = (jl < ncols && wj < wpr) ? col0 + jl : -1;
    if (jcol[c] >= 0) valid |= 1u << c;
  }
  const bool mycol = valid != 0;
  const int nq4 = (n_in + 3) >> 2;

  Lif lif;
  lif.load(d);
  const int vreset = FIXED ? d.Vreset : __float_as_int(d.vresetf);
  const int vinit = FIXED ? d.Vinit : __float_as_int(d.vinitf);
  const int t_ref = d.t_ref, t_inh = d.t_inh, t_ltp = d.t_ltp;
  const bool hard = d.wta_mode == 0;
  const bool stoch = d.stdp_mode == 0;
  const bool inh_reset = d.inh_mode == 0;
  const bool keep = (flags & FLAG_KEEP_STATE) != 0;
  const int tbase = keep ? d.t0 : 0;
  const int world = d.world;
  const bool sharded = world > 1;
  // epoch numbering of the shard exchange: continues the previous launch's count
  const uint32_t seq0 = sharded ? (uint32_t)ld_relaxed_sys_s32(reinterpret_cast<const int*>(&d.mbox->seq)) : 0u;

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
  int v[CPT], cnt[CPT], lpost[CPT];
#pragma unroll
  for (int c = 0; c < CPT; ++c) {
    v[c] = vinit; cnt[c] = 0; lpost[c] = kNever;
    if (keep && (valid >> c & 1u)) { v[c] = d.v[jcol[c]]; cnt[c] = d.cnt[jcol[c]]; lpost[c] = d.last_post[jcol[c]]; }
  }
  if (keep) for (int i = tid; i < n_in; i += nthr) s_lpre[i] = d.last_pre[i];
#pragma unroll
  for (int c = 0; c < CPT; ++c)
    if (valid >> c & 1u) s_lpost[jcol[c] - col0] = lpost[c];
  uint32_t ltd_trials = 0, ltd_events = 0, ltp_trials = 0, ltp_events = 0;   // per launch, < 2^32
  unsigned long long act_sum = 0, post_sum = 0;
  uint32_t eng_epochs = 0, eng_hz = 0, eng_resim = 0, eng_spec = 0, eng_undo = 0;
  if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }

  int ep = 0;
  unsigned long long* trace = d.trace ? d.trace + (size_t)rank * d.trace_cap * 8 : nullptr;
  unsigned long long* s_tmax = reinterpret_cast<unsigned long long*>(s_misc + 8);
  unsigned long long tr0 = 0, tr2 = 0, tr3 = 0;
  long long prof_int = 0, prof_ltd = 0, prof_seq = 0, prof_blk = 0, prof_loop0 = 0, prof_loop = 0;
  long long prof_ev = 0, prof_nev = 0;
  const long long prof_clk0 = clock64();
  const unsigned long long prof_ns0 = globaltimer();
  // pending LTP of the previous epoch (owner warps run it while the others start speculating)

  for (int b = 0; b < n_images; ++b) {
    const unsigned long long seed = d.seeds[b];
    if (!keep) {
#pragma unroll
      for (int c = 0; c < CPT; ++c) {
        v[c] = vinit; cnt[c] = 0; lpost[c] = kNever;
        if (valid >> c & 1u) s_lpost[jcol[c] - col0] = kNever;
      }
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
        __syncthreads();
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
        if (tid < 8) s_meta[nrows + tid] = (uint32_t)(n_in * wpr) | (0x1FFu << 16);   // zero-row pads
        // row metadata: word offset | window step (the link is added below)
        for (int x = tid; x < nsteps; x += nthr) {
          for (uint32_t r = s_offs[x] - wbase; r < s_offs[x + 1] - wbase; ++r)
            s_meta[r] = (uint32_t)s_rows[r] * (uint32_t)wpr | ((uint32_t)x << 16);
          // block starting at step x: nb = the most steps (<= kBlk, inside the window) holding <= 64 rows
          // in all (0: step x alone exceeds 64 rows -> general path), and which of them are non-empty
          const uint32_t o0 = s_offs[x];
          uint32_t nb = 0, ne = 0, prev = o0;
          for (int b = 0; b < kBlk && x + b < nsteps; ++b) {
            const uint32_t o = s_offs[x + b + 1];
            if (o - o0 > 64u) break;
            nb = b + 1;
            if (o != prev) ne |= 1u << b;
            prev = o;
          }
          s_binfo[x] = nb | (ne << 8);
        }
        __syncthreads();
        // link to the next occurrence of the same input within the next 64 rows and 8 steps (a block
        // holds <= 64 rows and <= kBlk steps; LTD sum corrections follow the links, block_correct)
        for (uint32_t r = tid; r < nrows; r += nthr) {
          const uint32_t mr = s_meta[r];
          const int x = meta_step(mr);
          const uint32_t id = s_rows[r];
          const uint32_t pat = id * 0x10001u;
          const uint32_t lim = min(min(nrows, r + 65u), s_offs[min(x + kBlk, nsteps)] - wbase);
          uint32_t link = 0;
          uint32_t y = r + 1;
          if (y & 1u) { if (y < lim && s_rows[y] == id) link = 1; ++y; }
          for (; !link && y < lim; y += 2) {   // two ids per 32-bit load (y + 1 <= rows_cap: allocated)
            const uint32_t eq = __vcmpeq2(*reinterpret_cast<const uint32_t*>(s_rows + y), pat);
            if (eq) { const uint32_t yy = y + ((eq & 0xFFFFu) ? 0u : 1u); if (yy < lim) link = yy - r; }
          }
          if (link) s_meta[r] = mr | (link << 25);
        }
        __syncthreads();
      }
      const int kend = kb;
      const int fp = ep & 1;
      const uint32_t cur = seq0 + (uint32_t)ep + 1u;        // shard-exchange epoch number (never 0 in use)
      if (trace && tid == 0) {
        tr0 = globaltimer(); *s_tmax = 0ull; s_misc[3] = 0;
        *reinterpret_cast<unsigned long long*>(s_misc + 10) = 0ull;
        *reinterpret_cast<unsigned long long*>(s_misc + 12) = 0ull;
      }

      // ---------------------------------------------------------- speculation (warp-synchronous, no CTA barrier)
      int p = kend;             // first step this thread did not fully process
      bool cand = false;        // stopped at a crossing at p (LIF done for all its columns, LTD pending)
      bool hz = false;          // stopped at p with nothing done (undo log full)
      uint32_t cmask = 0;       // columns crossing at p
      int cnt0[CPT], v1[CPT], cnt1[CPT], vb[CPT], cb[CPT];
#pragma unroll
      for (int c = 0; c < CPT; ++c) { cnt0[c] = cnt[c]; v1[c] = v[c]; cnt1[c] = cnt[c]; vb[c] = v[c]; cb[c] = cnt[c]; }
      int nlog = 0;
      {
        const uint32_t flag_addr = smem_u32(&s_flag[fp]);
        uint32_t ltd_cols = 0;                                    // columns with a valid last_post
#pragma unroll
        for (int c = 0; c < CPT; ++c)
          if (stoch && (valid >> c & 1u) && lpost[c] >= 0) ltd_cols |= 1u << c;
        bool done = !mycol;
        int kk = k0;
        int r0 = (int)(s_offs[k0 - ka] - wbase);
        auto signal = [&](int fstep) {                            // tell the cluster (and the other shards) where to stop
          atomicMin(&s_flag[fp], fstep);
          for (int r = 0; r < cs; ++r)
            if (r != rank) red_min_cluster(&s_flag[fp], (uint32_t)r, fstep);
          if (sharded) {
            const unsigned long long fv = ((unsigned long long)cur << 32) | (0xFFFFFFFFu - (uint32_t)fstep);
            for (int r = 0; r < world; ++r)
              if (r != d.shard) red_max_sys_u64(&d.peers[r]->flag, fv);
          }
        };
        // other shards' early-stop flag: lane 0 folds the value loaded one iteration earlier into the
        // CTA's flag and issues the next load (its latency overlaps the iteration)
        unsigned long long gflag_next = 0ull;
        if (sharded && lane == 0) gflag_next = ld_relaxed_sys_u64(&d.mbox->flag);
        long long e_int0 = prof_int, e_ltd0 = prof_ltd, e_seq0 = prof_seq, e_ev0 = prof_ev;
        if (trace && lane == 0) {
          prof_loop0 = clock64();
          const unsigned long long gt = globaltimer();
          atomicMax(reinterpret_cast<unsigned long long*>(s_misc + 10), gt);   // latest warp loop start
        }
        while (__any_sync(FULL, !done)) {
          if (sharded && lane == 0) {
            if ((uint32_t)(gflag_next >> 32) == cur) atomicMin(&s_flag[fp], (int)(0xFFFFFFFFu - (uint32_t)gflag_next));
            gflag_next = ld_relaxed_sys_u64(&d.mbox->flag);
          }
          __syncwarp();
          if (!done && (kk >= kend || kk > ld_volatile_shared_u32addr(flag_addr))) { done = true; p = kk; }
          if (kk >= kend) break;                                  // warp-uniform
          // ======== block path: up to kBlk steps of <= kPadRows rows each (<= 64 rows in all).
          // Integration of all block steps is independent of v, so it is issued at once from the
          // fixed-width row slots (pad index n_in -> the all-zero row); the block's LTD Philox blocks
          // are drawn in <= 2 warp-wide passes; only the LIF chain runs step by step.  An applied LTD
          // decrement at step b is subtracted from the sums of the later block steps that contain
          // the same row (exact: the sum was taken with the pre-decrement code).
          {
            const uint32_t bi = s_binfo[kk - ka];                // block shape (window staging)
            const int nb = (int)(bi & 0xFFu);
            const uint32_t nonempty = bi >> 8;                   // block steps with >= 1 active row
            if (nb > 0) {
              const int kb0 = kk;
              const bool prof = trace && lane == 0;
              long long pc0 = prof ? clock64() : 0;
              uint32_t* const my_acc = s_acc + tid;              // [b * nthr + tid]: SWAR sums of block step b
              const int rblk0 = r0;
              const int rblk1 = (int)(s_offs[kb0 - ka + nb] - wbase);
              // columns held (refractory / inhibited) through the whole block run no LIF, so their sums
              // are never used: a warp with no LIF and no LTD in the block only counts down (exact)
              uint32_t live = 0, ltd_pre = 0;
              if (!done) {
#pragma unroll
                for (int c = 0; c < CPT; ++c) {
                  if ((valid >> c & 1u) && cnt[c] < nb) live |= 1u << c;
                  if ((ltd_cols >> c & 1u) && (tbase + kb0 - lpost[c]) < L_dep) ltd_pre |= 1u << c;
                }
              }
              const bool warp_live = __any_sync(FULL, live != 0);
              if (!warp_live && !__any_sync(FULL, ltd_pre != 0)) {
                if (!done) {
                  int stop_at = nb;                                // honour the early-stop flag per step
                  const int f = ld_volatile_shared_u32addr(flag_addr);
                  if (f < kb0 + nb - 1) stop_at = max(1, f - kb0 + 1);
#pragma unroll
                  for (int c = 0; c < CPT; ++c) cnt[c] -= stop_at;
                  if (kb0 == k0) {
#pragma unroll
                    for (int c = 0; c < CPT; ++c) { v1[c] = v[c]; cnt1[c] = cnt[c] + stop_at - 1; }
                  }
                  if (stop_at < nb) { done = true; p = kb0 + stop_at; }
                }
                kk = kb0 + nb;
                r0 = rblk1;
                continue;
              }
              if (!done && warp_live) {
                // (a2) eq.(3) for all block steps in one flattened pass over the block's rows: the running
                // SWAR sum is stored into the slot of the row's step, so the slot of a non-empty step holds
                // the running sum at its end (lanes never overflow: <= 64 + 7 rows).  Branch-free groups of
                // 8 rows: rows past the block belong to later steps (or are zero-row pads) and land in
                // slots >= nb or the spill slot kBlk, which are never read.  All loads of a group are
                // issued before its stores (the slots share the buffer: the compiler would serialise).
                uint32_t run = 0u;
                const int sbase = kb0 - ka;
#pragma unroll 1
                for (int r = rblk0; r < rblk1; r += 8) {
                  uint32_t m[8], w[8];
#pragma unroll
                  for (int x = 0; x < 8; ++x) m[x] = s_meta[r + x];
#pragma unroll
                  for (int x = 0; x < 8; ++x) w[x] = (wcol[meta_woff(m[x])] >> fsh) & Z::LMASK;
#pragma unroll
                  for (int x = 0; x < 8; ++x) {
                    run += w[x];
                    my_acc[min(meta_step(m[x]) - sbase, kBlk) * nthr] = run;
                  }
                }
              }
              long long pc1 = prof ? clock64() : 0;
              // ---- LTD draws of the block for every LTD-active (lane, column) pair (eq.(7))
              uint32_t ltd_blk = 0;
              if (!done) {
#pragma unroll
                for (int c = 0; c < CPT; ++c)
                  if ((ltd_cols >> c & 1u) && (tbase + kb0 - lpost[c]) < L_dep) ltd_blk |= 1u << c;
              }
              const int nrows_blk = rblk1 - rblk0;
              if (SNN_EXP != 2 && __any_sync(FULL, ltd_blk != 0)) {
                // this lane's rows of the block and their steps (the same for every pair)
                const int bsel0 = lane < nrows_blk ? meta_step(s_meta[rblk0 + lane]) - (kb0 - ka) : 0;
                const int bsel1 = lane + 32 < nrows_blk ? meta_step(s_meta[rblk0 + 32 + lane]) - (kb0 - ka) : 0;
                const uint32_t row0 = lane < nrows_blk ? (uint32_t)s_rows[rblk0 + lane] : 0u;
                const uint32_t row1 = lane + 32 < nrows_blk ? (uint32_t)s_rows[rblk0 + 32 + lane] : 0u;
#pragma unroll 1
                for (uint32_t lm = __ballot_sync(FULL, ltd_blk != 0); lm; lm &= lm - 1) {
                  const int Ls = __ffs(lm) - 1;
                  const int tidL = warp * 32 + Ls;
#pragma unroll 1
                  for (uint32_t cm = __shfl_sync(FULL, ltd_blk, Ls); cm; cm &= cm - 1) {
                    const int c = __ffs(cm) - 1;
                    const int jlL = (tidL / TPW) * CPW + (tidL % TPW) + TPW * c;
                    const int jL = cbase + col0 + jlL;
                    const int lpL = s_lpost[jlL];
#pragma unroll 1
                    for (int m = 0; m < 2; ++m) {
                      const int x = 32 * m + lane;
                      bool bit = false;
                      if (x < nrows_blk) {
                        const int t = tbase + kb0 + (m ? bsel1 : bsel0);
                        const int D = t - lpL;
                        if (D < L_dep) {
                          const uint4 u = philox((uint32_t)t, m ? row1 : row0, (uint32_t)(jL >> 2), TAG_LTD, seed);
                          bit = pick(u, jL & 3) <= s_dep[D];
                        }
                      }
                      const uint32_t mm = __ballot_sync(FULL, bit);
                      if (lane == Ls) s_ev[(c * 2 + m) * nthr + tid] = mm;
                    }
                  }
                }
              }
              long long pc2 = prof ? clock64() : 0;
              // ---- this lane's LTD events of the block, once: 64-bit row masks per column and the block
              // steps that hold at least one event (the LIF chain below only branches on those)
              unsigned long long e64c[CPT];
              uint32_t evsteps = 0u;
#pragma unroll
              for (int c = 0; c < CPT; ++c) {
                e64c[c] = 0ull;
                if (SNN_EXP != 2 && (ltd_blk >> c & 1u)) {
                  e64c[c] = (unsigned long long)s_ev[(c * 2) * nthr + tid] |
                            ((unsigned long long)s_ev[(c * 2 + 1) * nthr + tid] << 32);
                  for (unsigned long long m = e64c[c]; m; m &= m - 1ull)
                    evsteps |= 1u << (meta_step(s_meta[rblk0 + __ffsll((long long)m) - 1]) - (kb0 - ka));
                }
              }
              // ---- sequential LIF over the block (the only step-to-step dependency)
              if (!done) {
                uint32_t run_prev = 0u;
                int bdone = nb;                                      // block steps committed by this lane
                // software pipelined: the next step's sum slot and the early-stop flag are loaded one step
                // ahead (a flag seen one step late only speculates one step further, which the resolution
                // rolls back like any overrun)
                uint32_t slot_nx = my_acc[0];
                int flag_nx = INT_MAX;
#pragma unroll 1
                for (int b = 0; b < nb; ++b) {
                  const int kk_b = kb0 + b;
                  // a crossing before kk_b exists in the cluster: stop here (state is that after kk_b - 1)
                  if (b > 0 && kk_b > flag_nx) { done = true; p = kk_b; bdone = b; break; }
                  const uint32_t snap = (nonempty >> b & 1u) ? slot_nx : run_prev;
                  if (b + 1 < nb) slot_nx = my_acc[(b + 1) * nthr];
                  flag_nx = ld_volatile_shared_u32addr(flag_addr);
                  const uint32_t a = snap - run_prev;              // this step's SWAR sums
                  run_prev = snap;
                  uint32_t cm_b = 0;
                  int vn[CPT];
#pragma unroll
                  for (int c = 0; c < CPT; ++c) {                     // branch-free: the CPT chains overlap
                    const int S = (int)(Z::LW == 32 ? a : ((a >> (c * Z::LW)) & ((1u << (Z::LW & 31)) - 1u)));
                    vn[c] = v[c];
                    const bool crossed = lif.step_t<FIXED>(vn[c], S);
                    cm_b |= ((cnt[c] == 0 && crossed && (valid >> c & 1u)) ? 1u : 0u) << c;
                  }
                  if (cm_b) {                                         // stop here: LIF done, LTD pending
#pragma unroll
                    for (int c = 0; c < CPT; ++c) {
                      cb[c] = cnt[c]; vb[c] = v[c];
                      v[c] = cnt[c] == 0 ? vn[c] : v[c];
                      cnt[c] = cnt[c] == 0 ? 0 : cnt[c] - 1;
                    }
                    cmask = cm_b; cand = true; done = true; p = kk_b; bdone = b; signal(kk_b);
                    break;
                  }
                  const long long pe0 = prof ? clock64() : 0;
                  if (SNN_EXP != 1 && (evsteps >> b & 1u)) {          // LTD events of step b (rare)
                    const int rlo = (int)(s_offs[kk_b - ka] - wbase), rhi = (int)(s_offs[kk_b - ka + 1] - wbase);
                    const int lo = rlo - rblk0, nrb = rhi - rlo;
                    const int nlog_step = nlog;
                    bool overflow = false;
                    uint32_t ev_step = 0;
#pragma unroll
                    for (int c = 0; c < CPT; ++c) {
                      if (overflow || !(ltd_blk >> c & 1u)) continue;
                      unsigned long long em = nrb ? ((e64c[c] >> lo) & ((1ull << nrb) - 1ull)) : 0ull;
                      const int shc = fsh + c * Z::LW;
                      while (em) {
                        const int xr = __ffsll((long long)em) - 1;
                        em &= em - 1;
                        if (kk_b > k0 && nlog == logn) { overflow = true; break; }
                        const int i = s_rows[rlo + xr];
                        uint32_t* pw = wcol + i * wpr;
                        const bool applied = ((*pw >> shc) & FMASK) != 0u;
                        if (applied) {
                          atomicSub(pw, 1u << shc);
                          // the later block steps that contain row i were summed with the old code
                          if (meta_link(s_meta[rlo + xr]))
                            block_correct(s_meta, my_acc, nthr, rlo + xr, rblk1, kb0 - ka, nonempty, 0u - (1u << (c * Z::LW)));
                        }
                        ++ev_step;
                        if (kk_b > k0) s_log[nlog++ * nthr + tid] = log_entry(kk_b - k0, c, applied, i);
                      }
                    }
                    if (overflow) {                               // undo step b entirely; stop before it
                      while (nlog > nlog_step) {
                        const uint32_t e = s_log[(nlog - 1) * nthr + tid];
                        const int i = (int)(e & 0x1FFFu), c = (int)((e >> 14) & 3u);
                        if (e & 0x2000u) {
                          atomicAdd(wcol + i * wpr, 1u << (fsh + c * Z::LW));
                          int rpos = rlo;                             // the event's row position in step b
                          while (rpos < rhi - 1 && (int)s_rows[rpos] != i) ++rpos;
                          block_correct(s_meta, my_acc, nthr, rpos, rblk1, kb0 - ka, nonempty, 1u << (c * Z::LW));
                        }
                        --nlog;
                      }
                      hz = true; done = true; p = kk_b; bdone = b; ++eng_hz;   // v / cnt of step b were not committed
                      signal(kk_b - 1);
                      break;
                    }
                    ltd_events += ev_step;
                    if (trace) prof_nev += ev_step;
                    if (b + 1 < nb) slot_nx = my_acc[(b + 1) * nthr];   // the corrections may have changed it
                  }
                  if (prof) { __syncwarp(__activemask()); prof_ev += clock64() - pe0; }
#pragma unroll
                  for (int c = 0; c < CPT; ++c) {                     // commit step b
                    v[c] = cnt[c] == 0 ? vn[c] : v[c];
                    cnt[c] = cnt[c] == 0 ? 0 : cnt[c] - 1;
                  }
                  if (kk_b == k0) {
#pragma unroll
                    for (int c = 0; c < CPT; ++c) { v1[c] = v[c]; cnt1[c] = cnt[c]; }
                  }
                }
                // LTD trials of the committed block steps: rows of steps b < bdone with D = t - last_post < L_dep
                if (ltd_blk) {
#pragma unroll
                  for (int c = 0; c < CPT; ++c) {
                    if (!(ltd_blk >> c & 1u)) continue;
                    const int blim = min(bdone, lpost[c] + L_dep - tbase - kb0);
                    if (blim > 0) ltd_trials += s_offs[kb0 - ka + blim] - s_offs[kb0 - ka];
                  }
                }
              }
              if (prof) {
                const long long pc3 = clock64();
                prof_int += pc1 - pc0; prof_ltd += pc2 - pc1; prof_seq += pc3 - pc2; prof_blk += nb;
              }
              kk = kb0 + nb;
              r0 = rblk1;
              continue;
            }
          }
          // ======== general path: one step (more than kPadRows active rows)
          const int r1 = (int)(s_offs[kk - ka + 1] - wbase);
          const int t = tbase + kk;
          uint32_t ltd_on = 0;
          if (!done) {
            int S[CPT];
            integrate_swar<BITS, CPT>(wcol, s_rows, r0, r1, wpr, fsh, S);        // (a2) eq.(3)
#pragma unroll
            for (int c = 0; c < CPT; ++c) {
              cb[c] = cnt[c];
              if (!(valid >> c & 1u)) continue;
              if (cnt[c] > 0) {
                --cnt[c];                                         // (a3) refractory / inhibited: hold v
              } else {
                vb[c] = v[c];
                if (lif.step_t<FIXED>(v[c], S[c])) cmask |= 1u << c;   // (a3) eqs.(1)(2)
              }
            }
            if (cmask) { cand = true; done = true; p = kk; signal(kk); }
            else {
#pragma unroll
              for (int c = 0; c < CPT; ++c)
                if ((ltd_cols >> c & 1u) && (t - lpost[c]) < L_dep) ltd_on |= 1u << c;
            }
          }
          // (a5) LTD, eq.(7), exact (R10, R14): for every LTD-active (lane, column) pair of the warp,
          // all 32 lanes draw the Philox blocks of up to 32 active rows at once (one rolled call site
          // keeps the loop inside the instruction cache); the owning lane applies its events.
          if (__any_sync(FULL, ltd_on != 0)) {
            const int nlog_step = nlog;
            bool overflow = false;
            uint32_t ev_step = 0;
#pragma unroll 1
            for (uint32_t lm = __ballot_sync(FULL, ltd_on != 0); lm; lm &= lm - 1) {
              const int Ls = __ffs(lm) - 1;
              const int tidL = warp * 32 + Ls;
#pragma unroll 1
              for (uint32_t cm = __shfl_sync(FULL, ltd_on, Ls); cm; cm &= cm - 1) {
                const int c = __ffs(cm) - 1;
                const int jlL = (tidL / TPW) * CPW + (tidL % TPW) + TPW * c;
                const int jL = cbase + col0 + jlL;
                const uint32_t thrL = s_dep[t - s_lpost[jlL]];
                const int shc = fsh + c * Z::LW;
#pragma unroll 1
                for (int c0 = r0; c0 < r1; c0 += 32) {
                  const int n = min(32, r1 - c0);
                  bool bit = false;
                  if (lane < n) {
                    const uint4 u = philox((uint32_t)t, (uint32_t)s_rows[c0 + lane], (uint32_t)(jL >> 2), TAG_LTD, seed);
                    bit = pick(u, jL & 3) <= thrL;
                  }
                  uint32_t mine = __ballot_sync(FULL, bit);
                  if (lane == Ls) {
                    while (mine && !overflow) {
                      const int x = __ffs(mine) - 1;
                      mine &= mine - 1;
                      if (kk > k0 && nlog == logn) { overflow = true; break; }
                      const int i = s_rows[c0 + x];
                      uint32_t* pw = wcol + i * wpr;
                      const bool applied = ((*pw >> shc) & FMASK) != 0u;
                      if (applied) atomicSub(pw, 1u << shc);
                      ++ev_step;
                      if (kk > k0) s_log[nlog++ * nthr + tid] = log_entry(kk - k0, c, applied, i);
                    }
                  }
                }
              }
            }
            if (ltd_on) {
              if (overflow) {                                      // undo this step entirely; stop before it
                while (nlog > nlog_step) {
                  const uint32_t e = s_log[(nlog - 1) * nthr + tid];
                  if (e & 0x2000u) atomicAdd(wcol + (int)(e & 0x1FFFu) * wpr, 1u << (fsh + (int)((e >> 14) & 3u) * Z::LW));
                  --nlog;
                }
#pragma unroll
                for (int c = 0; c < CPT; ++c) { if (cb[c] == 0) v[c] = vb[c]; cnt[c] = cb[c]; }
                hz = true;
                done = true;
                p = kk;
                ++eng_hz;
                signal(kk - 1);
              } else {
                ltd_events += ev_step;
                ltd_trials += (uint32_t)__popc(ltd_on) * (uint32_t)(r1 - r0);
              }
            }
          }
          if (!done && kk == k0) {
#pragma unroll
            for (int c = 0; c < CPT; ++c) { v1[c] = v[c]; cnt1[c] = cnt[c]; }
          }
          ++kk;
          r0 = r1;
        }
        if (trace && lane == 0) {
          const long long dl = clock64() - prof_loop0;
          prof_loop += dl;
          atomicMax(reinterpret_cast<unsigned long long*>(s_misc + 12), (unsigned long long)dl);  // longest warp loop
          // per-warp per-epoch breakdown (16-bit fields, cycles/16): int | ltd | seq | events
          unsigned long long* s_wp = reinterpret_cast<unsigned long long*>(s_misc + 16 + nthr * CPT + 4) + warp * 2;
          s_wp[0] = (unsigned long long)dl;
          s_wp[1] = (unsigned long long)(min((prof_int - e_int0) >> 4, 0xFFFFll)) |
                    ((unsigned long long)(min((prof_ltd - e_ltd0) >> 4, 0xFFFFll)) << 16) |
                    ((unsigned long long)(min((prof_seq - e_seq0) >> 4, 0xFFFFll)) << 32) |
                    ((unsigned long long)(min((prof_ev - e_ev0) >> 4, 0xFFFFll)) << 48);
        }
        if (!mycol) p = kend;
        if (mycol) eng_spec += (uint32_t)(p - k0 + (cand ? 1 : 0)) * (uint32_t)__popc(valid);
      }
      if (trace && lane == 0) atomicMax(s_tmax, globaltimer());
      if (trace && mycol) atomicMax(&s_misc[3], p - k0);       // deepest speculation of the CTA

      // ---------------------------------------------------------- CTA summary -> cluster exchange
      {
        const uint32_t w1 = ((uint32_t)(0xFFFF - min(p, kend)) << 1) | (hz ? 1u : 0u);
        const uint32_t W1w = __reduce_max_sync(FULL, w1);
        const int Pw = 0xFFFF - (int)(W1w >> 1);
        const bool c_at = cand && p == Pw;
        uint32_t kh = 0, kl = 0, cc = 0;
        if (c_at) {
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            if (!(cmask >> c & 1u)) continue;
            const uint32_t h = lif.ord(v[c]), l = 0xFFFFFFFFu - (uint32_t)(jcol[c] + cbase);
            if (h > kh || (h == kh && l > kl)) { kh = h; kl = l; }
            ++cc;
          }
        }
        const uint32_t mh = __reduce_max_sync(FULL, kh);
        const uint32_t ml = __reduce_max_sync(FULL, (c_at && kh == mh) ? kl : 0u);
        const uint32_t cw = __reduce_add_sync(FULL, cc);
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
        const uint32_t ccs = __reduce_add_sync(FULL, at ? (uint32_t)a : 0u);
        const uint32_t kh = __reduce_max_sync(FULL, at ? (uint32_t)(k >> 32) : 0u);
        const uint32_t kl = __reduce_max_sync(FULL, (at && (uint32_t)(k >> 32) == kh) ? (uint32_t)k : 0u);
        const unsigned long long A = ((unsigned long long)W1c << 32) | ccs;
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
      uint32_t W1, count;
      unsigned long long K;
      {                                                    // lane r reads CTA r's summary; warp reductions
        const unsigned long long A = lane < cs ? s_slots[(size_t)(fp * kMaxCluster + lane) * 2] : 0ull;
        const unsigned long long Kr = lane < cs ? s_slots[(size_t)(fp * kMaxCluster + lane) * 2 + 1] : 0ull;
        W1 = __reduce_max_sync(FULL, (uint32_t)(A >> 32));
        const bool at = lane < cs && (uint32_t)(A >> 32) == W1;
        count = __reduce_add_sync(FULL, at ? (uint32_t)A : 0u);
        const uint32_t kh = __reduce_max_sync(FULL, at ? (uint32_t)(Kr >> 32) : 0u);
        const uint32_t kl = __reduce_max_sync(FULL, (at && (uint32_t)(Kr >> 32) == kh) ? (uint32_t)Kr : 0u);
        K = ((unsigned long long)kh << 32) | kl;
      }
      if (sharded) {
        // (e) column sharding: the cluster's summary {A, K} goes to slot [cur & 1][shard] of every rank's
        // mailbox as four LL words (NVLink peer stores); warp 0 of every CTA reads the world's summaries
        // from its own mailbox and applies the same reduction as the cluster exchange
        const int mp = (int)(cur & 1u);
        const unsigned long long tag = (unsigned long long)cur << 32;
        if (rank == 0 && warp == 0 && lane < world) {           // lane r -> rank r: four LL words, no fence
          unsigned long long* sl = d.peers[lane]->slot[mp][d.shard];
          st_relaxed_sys_u64(sl, tag | W1);
          st_relaxed_sys_u64(sl + 1, tag | count);
          st_relaxed_sys_u64(sl + 2, tag | (uint32_t)(K >> 32));
          st_relaxed_sys_u64(sl + 3, tag | (uint32_t)K);
        }
        if (warp == 0) {                                           // warp 0 polls; the CTA reads its result
          unsigned long long A = 0ull, Kr = 0ull;
          if (lane < world) {
            const unsigned long long* sl = d.mbox->slot[mp][lane];
            const unsigned long long t_start = globaltimer();
            unsigned long long w0, w1, w2, w3;
            while (true) {
              w0 = ld_relaxed_sys_u64(sl); w1 = ld_relaxed_sys_u64(sl + 1);
              w2 = ld_relaxed_sys_u64(sl + 2); w3 = ld_relaxed_sys_u64(sl + 3);
              if ((uint32_t)(w0 >> 32) == cur && (uint32_t)(w1 >> 32) == cur && (uint32_t)(w2 >> 32) == cur &&
                  (uint32_t)(w3 >> 32) == cur) break;
              if (globaltimer() - t_start > kShardTimeoutNs) __trap();   // a rank is gone: fail, never hang
            }
            A = ((unsigned long long)(uint32_t)w0 << 32) | (uint32_t)w1;
            Kr = ((unsigned long long)(uint32_t)w2 << 32) | (uint32_t)w3;
          }
          const uint32_t W1g = __reduce_max_sync(FULL, (uint32_t)(A >> 32));
          const bool at = lane < world && (uint32_t)(A >> 32) == W1g;
          const uint32_t cg = __reduce_add_sync(FULL, at ? (uint32_t)A : 0u);
          const uint32_t kh = __reduce_max_sync(FULL, at ? (uint32_t)(Kr >> 32) : 0u);
          const uint32_t kl = __reduce_max_sync(FULL, (at && (uint32_t)(Kr >> 32) == kh) ? (uint32_t)Kr : 0u);
          if (lane == 0) {     // s_wsum is free here: the CTA summary was consumed before the cluster exchange
            s_wsum[0] = ((unsigned long long)W1g << 32) | cg;
            s_wsum[1] = ((unsigned long long)kh << 32) | kl;
          }
        }
        __syncthreads();
        W1 = (uint32_t)(s_wsum[0] >> 32);
        count = (uint32_t)s_wsum[0];
        K = s_wsum[1];
        if (trace && tid == 0) tr3 = globaltimer();            // sharded: "exchanged" = after the world exchange
      }
      const int P = 0xFFFF - (int)(W1 >> 1);
      const bool unknown = (W1 & 1u) != 0u;
      const bool at_end = P >= kend;
      const bool event = !at_end && !unknown;
      const int tP = tbase + P;

      // ---------------------------------------------------------- per-thread resolution / rollback
      auto count_trials = [&](int c, int from, int to) -> uint32_t {   // LTD trials of column c, steps [from, to)
        if (!stoch || lpost[c] < 0) return 0u;
        const int last = lpost[c] + L_dep - 1 - tbase;                 // last step with D < L_dep
        const int hi = min(to, last + 1);
        return hi > from ? s_offs[hi - ka] - s_offs[from - ka] : 0u;
      };
      auto undo_after = [&](int rel_keep) {       // undo logged LTD of steps k0 + rel > k0 + rel_keep
        while (nlog > 0) {
          const uint32_t e = s_log[(nlog - 1) * nthr + tid];
          if ((int)(e >> 16) <= rel_keep) break;
          if (e & 0x2000u) atomicAdd(wcol + (int)(e & 0x1FFFu) * wpr, 1u << (fsh + (int)((e >> 14) & 3u) * Z::LW));
          --ltd_events;
          --nlog;
          ++eng_undo;
        }
      };
      // per-lane LTD of all this thread's LTD-active columns at step kk (commit / re-simulation paths)
      auto ltd_step = [&](int kk) {
        const int t = tbase + kk;
        const int r0 = (int)(s_offs[kk - ka] - wbase), r1 = (int)(s_offs[kk - ka + 1] - wbase);
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
          if (!stoch || !(valid >> c & 1u) || lpost[c] < 0 || (t - lpost[c]) >= L_dep) continue;
          const uint32_t thr = s_dep[t - lpost[c]];
          const int shc = fsh + c * Z::LW;
          for (int r = r0; r < r1; ++r) {
            const int i = s_rows[r];
            const int jg = jcol[c] + cbase;
            const uint4 u = philox((uint32_t)t, (uint32_t)i, (uint32_t)(jg >> 2), TAG_LTD, seed);
            if (pick(u, jg & 3) <= thr) {
              uint32_t* pw = wcol + i * wpr;
              if ((*pw >> shc) & FMASK) atomicSub(pw, 1u << shc);
              ++ltd_events;
            }
          }
          ltd_trials += (uint32_t)(r1 - r0);
        }
      };
      auto resim = [&](int X) {      // state after step k0, undo every logged LTD, replay k0+1 .. X exactly
        ++eng_resim;
        undo_after(0);
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
          ltd_trials -= count_trials(c, k0 + 1, p);
          v[c] = v1[c]; cnt[c] = cnt1[c];
        }
        for (int kk = k0 + 1; kk <= X; ++kk) {
          const int r0 = (int)(s_offs[kk - ka] - wbase), r1 = (int)(s_offs[kk - ka + 1] - wbase);
          int S[CPT];
          integrate_swar<BITS, CPT>(wcol, s_rows, r0, r1, wpr, fsh, S);
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            if (!(valid >> c & 1u)) continue;
            if (cnt[c] > 0) --cnt[c]; else lif.step_t<FIXED>(v[c], S[c]);
          }
          ltd_step(kk);
        }
      };
      if (mycol && !at_end) {
        if (event) {
          if (p > P) {                                   // ran past t*: rebuild the state after step t*
            if (inh_reset) {
              undo_after(P - k0);
#pragma unroll
              for (int c = 0; c < CPT; ++c) {
                ltd_trials -= count_trials(c, P + 1, p);
                cnt[c] = max(cnt0[c] - (P - k0 + 1), 0);  // no crossing in [k0, t*]: cnt only counted down
              }
            } else {
              resim(P);
            }
          }
        } else {                                         // unknown at P: commit only through P - 1
          if (p == P) {
            if (cand) {
#pragma unroll
              for (int c = 0; c < CPT; ++c) { if (cb[c] == 0) v[c] = vb[c]; cnt[c] = cb[c]; }
            }
          } else {
            resim(P - 1);
          }
        }
      }
      uint32_t spiked = 0;
      if (event) {
        const uint32_t W = 0xFFFFFFFFu - (uint32_t)K;
        const bool at_p = cand && p == P;
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
          if (!(valid >> c & 1u)) continue;
          bool me;
          if (hard) me = (uint32_t)(jcol[c] + cbase) == W;
          else me = at_p && (cmask >> c & 1u);
          if (me) { v[c] = vreset; cnt[c] = t_ref; spiked |= 1u << c; }
          if (hard ? !me : (count >= 2u || !me)) { cnt[c] = max(cnt[c], t_inh); if (inh_reset) v[c] = vreset; }
        }
        img_spikes += hard ? 1 : (int)count;
        // pending LTD at t* of the columns that stopped there (old last_post, R14): warp-cooperative draws
        if (__any_sync(FULL, mycol && at_p)) {
          const int r0 = (int)(s_offs[P - ka] - wbase), r1 = (int)(s_offs[P - ka + 1] - wbase);
          uint32_t on = 0;
          if (mycol && at_p) {
#pragma unroll
            for (int c = 0; c < CPT; ++c)
              if (stoch && (valid >> c & 1u) && lpost[c] >= 0 && (tP - lpost[c]) < L_dep) on |= 1u << c;
          }
#pragma unroll 1
          for (uint32_t lm = __ballot_sync(FULL, on != 0); lm; lm &= lm - 1) {
            const int Ls = __ffs(lm) - 1;
            const int tidL = warp * 32 + Ls;
#pragma unroll 1
            for (uint32_t cm = __shfl_sync(FULL, on, Ls); cm; cm &= cm - 1) {
              const int c = __ffs(cm) - 1;
              const int jlL = (tidL / TPW) * CPW + (tidL % TPW) + TPW * c;
              const int jL = cbase + col0 + jlL;
              const uint32_t thrL = s_dep[tP - s_lpost[jlL]];
              const int shc = fsh + c * Z::LW;
#pragma unroll 1
              for (int c0 = r0; c0 < r1; c0 += 32) {
                const int n = min(32, r1 - c0);
                bool bit = false;
                if (lane < n) {
                  const uint4 u = philox((uint32_t)tP, (uint32_t)s_rows[c0 + lane], (uint32_t)(jL >> 2), TAG_LTD, seed);
                  bit = pick(u, jL & 3) <= thrL;
                }
                uint32_t mine = __ballot_sync(FULL, bit);
                if (lane == Ls) {
                  while (mine) {
                    const int x = __ffs(mine) - 1;
                    mine &= mine - 1;
                    uint32_t* pw = wcol + (int)s_rows[c0 + x] * wpr;
                    if ((*pw >> shc) & FMASK) atomicSub(pw, 1u << shc);
                    ++ltd_events;
                  }
                }
              }
              if (lane == Ls) ltd_trials += (uint32_t)(r1 - r0);
            }
          }
        }
        if (rec_out && spiked) {
#pragma unroll
          for (int c = 0; c < CPT; ++c)
            if (spiked >> c & 1u) atomicOr(&d.raster_out[(size_t)P * nwe + (jcol[c] >> 5)], 1u << (jcol[c] & 31));
        }
      }
      if (event && spiked) {                               // this CTA's spikers (local column index)
#pragma unroll
        for (int c = 0; c < CPT; ++c)
          if (spiked >> c & 1u) { const int pos = atomicAdd(&s_misc[1], 1); s_misc[16 + pos] = jcol[c] - col0; }
      }
      const int k_last = event ? P : (at_end ? kend - 1 : P - 1);
      // spike timers of the inputs through the committed step
      for (int kk = k0 + tid; kk <= k_last; kk += nthr) {
        const int r0 = (int)(s_offs[kk - ka] - wbase), r1 = (int)(s_offs[kk - ka + 1] - wbase);
        for (int r = r0; r < r1; ++r) atomicMax(&s_lpre[s_rows[r]], tbase + kk);
      }
      __syncthreads();                                                               // S2
      if (trace && tid == 0 && ep < d.trace_cap) {
        unsigned long long* rec = trace + (size_t)ep * 8;
        rec[0] = ((unsigned long long)b << 32) | (unsigned)k0;
        rec[1] = ((unsigned long long)(event ? 1 : (unknown ? 2 : 0)) << 32) | (unsigned)P;
        unsigned long long best = 0, bestw = 0;
        {
          const unsigned long long* s_wp = reinterpret_cast<const unsigned long long*>(s_misc + 16 + nthr * CPT + 4);
          for (int w = 0; w < nwarps; ++w) if (s_wp[2 * w] > best) { best = s_wp[2 * w]; bestw = s_wp[2 * w + 1]; }
        }
        rec[2] = tr0; rec[3] = *s_tmax; rec[4] = bestw; rec[5] = tr3;
        rec[6] = (unsigned long long)s_misc[3] |
                 ((*reinterpret_cast<unsigned long long*>(s_misc + 12)) << 16);   // depth | longest warp loop (cycles)
        rec[7] = globaltimer();
      }
      if (spiked) {
#pragma unroll
        for (int c = 0; c < CPT; ++c)
          if (spiked >> c & 1u) { lpost[c] = tP; s_lpost[jcol[c] - col0] = tP; }
      }
      // (a5) LTP eq.(6) / (a6) deterministic arm eqs.(4)(5)(8) at t* for this CTA's spikers: every thread
      // takes (spiker, group of 4 rows) pairs; updates are atomic (two spikers may share a row word)
      const int nsp = event ? s_misc[1] : 0;
      if (nsp > 0) {
        for (int item = tid; item < nsp * nq4; item += nthr) {
          const int m = item / nq4, grp = item - m * nq4;
          const int jl = s_misc[16 + m];
          const int Wg = cbase + col0 + jl;
          const int ww = jl / CPW, wsh = (jl % CPW) * BITS;
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
              if (pick(u, r) <= s_pot[D]) {                    // eq.(6), R10: Dt = D >= 0
                ++ltp_events;
                if (((*pw >> wsh) & FMASK) < (uint32_t)qmax) atomicAdd(pw, 1u << wsh);
              }
            } else {                                           // eqs.(4)(5)(8), R16/R17
              const int q0 = (int)((*pw >> wsh) & FMASK);
              const bool pot = lpi >= 0 && (tP - lpi) <= t_ltp;
              const int base = pot ? s_dbp[q0] : s_dbd[q0];
              const uint32_t thr = pot ? s_dtp[q0] : s_dtd[q0];
              const int dq = base + (pick(u, r) < thr ? 1 : 0);
              int q1 = pot ? q0 + dq : q0 - dq;
              q1 = q1 < 0 ? 0 : (q1 > qmax ? qmax : q1);
              if (q1 != q0) atomicAdd(pw, (uint32_t)(q1 - q0) << wsh);
              if (pot) { ++ltp_trials; if (dq > 0) ++ltp_events; }
              else     { ++ltd_trials; if (dq > 0) ++ltd_events; }
            }
          }
        }
        __syncthreads();                                                             // S4
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
#pragma unroll
      for (int c = 0; c < CPT; ++c)
        if (valid >> c & 1u) { d.v[jcol[c]] = v[c]; d.cnt[jcol[c]] = cnt[c]; d.last_post[jcol[c]] = lpost[c]; }
      __syncthreads();
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
  // slowest warp of the CTA (by whole speculation-loop cycles) reports its phase profile
  if (trace) {
    __syncthreads();
    unsigned long long* s_pm = reinterpret_cast<unsigned long long*>(s_misc + 8);
    if (tid == 0) *s_pm = 0ull;
    __syncthreads();
    if (lane == 0) atomicMax(s_pm, ((unsigned long long)prof_loop << 8) | (unsigned)warp);
    prof_nev = __reduce_add_sync(FULL, (unsigned)prof_nev);
    __syncthreads();
    if (lane == 0 && (int)(*s_pm & 0xFFull) == warp && d.trace_cap > 0) {
      unsigned long long* rec = trace + (size_t)(d.trace_cap - 1) * 8;
      rec[0] = (0xFFFFFFFFull << 32) | ((unsigned long long)(prof_nev & 0xFFFF) << 16) | (unsigned)warp;
      rec[1] = (unsigned long long)prof_int;
      rec[2] = (unsigned long long)prof_ltd; rec[3] = (unsigned long long)prof_seq; rec[4] = (unsigned long long)prof_blk;
      rec[5] = (unsigned long long)prof_loop; rec[6] = (unsigned long long)prof_ev;
      rec[7] = globaltimer() - prof_ns0;
    }
  }
  if (false) {
    unsigned long long* rec = trace + (size_t)(d.trace_cap - 1) * 8;
    rec[0] = 0xFFFFFFFFull << 32; rec[1] = (unsigned long long)prof_int; rec[2] = (unsigned long long)prof_ltd;
    rec[3] = (unsigned long long)prof_seq; rec[4] = (unsigned long long)prof_blk; rec[5] = (unsigned long long)prof_loop;
    rec[6] = (unsigned long long)(clock64() - prof_clk0); rec[7] = globaltimer() - prof_ns0;
  }
  if (cs > 1) { cluster_arrive(); cluster_wait(); }
  else if (sharded) __syncthreads();
  if (sharded && rank == 0 && tid == 0) d.mbox->seq = seq0 + (uint32_t)ep;   // every CTA read seq0 long ago
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
                           long long rows_stride, uint32_t* offs, uint16_t* rows, uint16_t* rows16, cudaStream_t s) {
  if (n_images <= 0) return cudaSuccess;
  compact_kernel<<<(unsigned)n_images, 256, 0, s>>>(words, counts, n_in, T, rows_stride, offs, rows, rows16);
  return cudaGetLastError();
}

template <int BITS, int CPT, bool FIXED>
static cudaError_t configure_event_t(size_t smem, int cs) {
  cudaError_t e = cudaFuncSetAttribute(present_event_kernel<BITS, CPT, FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (cs > 8) e = cudaFuncSetAttribute(present_event_kernel<BITS, CPT, FIXED>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
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

template <int BITS, int CPT, bool FIXED>
static cudaError_t launch_t(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, cudaStream_t s,
                            int* occupancy_out) {
  cudaError_t e = configure_event_t<BITS, CPT, FIXED>(smem, cs);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg;
  cudaLaunchAttribute attr[1];
  fill_cfg_ev(cfg, attr, n_nets, cs, nthr, smem, s);
  if (occupancy_out) {
    if (cs == 1) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occupancy_out, present_event_kernel<BITS, CPT, FIXED>, nthr, smem);
    return cudaOccupancyMaxActiveClusters(occupancy_out, present_event_kernel<BITS, CPT, FIXED>, &cfg);
  }
  return cudaLaunchKernelEx(&cfg, present_event_kernel<BITS, CPT, FIXED>, lp);
}

template <int BITS, int CPT>
static cudaError_t dispatch_f(int fixed, const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem,
                              cudaStream_t s, int* occ) {
  return fixed ? launch_t<BITS, CPT, true>(lp, n_nets, cs, nthr, smem, s, occ)
               : launch_t<BITS, CPT, false>(lp, n_nets, cs, nthr, smem, s, occ);
}

static cudaError_t dispatch(int bits, int cpt, int fixed, const LaunchParams& lp, int n_nets, int cs, int nthr,
                            size_t smem, cudaStream_t s, int* occ) {
  if (bits == 2) {
    if (cpt == 4) return dispatch_f<2, 4>(fixed, lp, n_nets, cs, nthr, smem, s, occ);
    if (cpt == 1) return dispatch_f<2, 1>(fixed, lp, n_nets, cs, nthr, smem, s, occ);
    return dispatch_f<2, 2>(fixed, lp, n_nets, cs, nthr, smem, s, occ);
  }
  if (bits == 4) {
    if (cpt == 1) return dispatch_f<4, 1>(fixed, lp, n_nets, cs, nthr, smem, s, occ);
    return dispatch_f<4, 2>(fixed, lp, n_nets, cs, nthr, smem, s, occ);
  }
  return dispatch_f<8, 1>(fixed, lp, n_nets, cs, nthr, smem, s, occ);
}

int event_threads(int max_groups, int bits, int cpt) {
  const int t = max_groups * 32 / cpt;            // CPW/CPT threads per packed word
  return ((t + 31) / 32) * 32;
}

cudaError_t query_max_clusters_event(int bits, int cpt, int fixed, int cs, int nthr, size_t smem, int* out) {
  LaunchParams lp{};
  return dispatch(bits, cpt, fixed, lp, 1, cs, nthr, smem, 0, out);
}

cudaError_t launch_present_event_mode(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, int bits,
                                      int cpt, int fixed, cudaStream_t s) {
  return dispatch(bits, cpt, fixed, lp, n_nets, cs, nthr, smem, s, nullptr);
}

}  // namespace snn
