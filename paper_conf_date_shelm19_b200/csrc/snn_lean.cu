// snn_lean.cu -- lean event-engine kernel for the paper's default learning mode:
// HARD winner-take-all with RESET inhibition (R7) and stochastic 1-LSB STDP (eqs.(6)(7),
// P:89).  Same epoch protocol as snn_event.cu (one cluster exchange per post-spike epoch; the
// columns run ahead independently between spikes), restructured around what that mode makes true:
//   * after every post spike EVERY column restarts from a state fixed by its own countdown
//     (v <- v_reset, cnt <- max(cnt, t_inh), the winner cnt <- t_ref), so a column that ran past the
//     first crossing t* is rebuilt in O(1) -- no membrane snapshot, no re-simulation;
//   * LTD of a column depends only on its own last_post and the input raster (R10, R14), so the
//     Philox draws of a warp's LTD-active columns are taken for 32 upcoming input rows at once
//     (lanes over rows), off the LIF chain; the decrements are applied in step order as the chain
//     reaches them, so every integration reads the codes of its own step and no sum is ever corrected;
//   * integration is inline per step from a padded row list (one 16-byte load yields 4 row offsets),
//     summing the thread's CPT columns in SWAR lanes (eq.(3)); held (refractory / inhibited) warps skip
//     whole runs of steps in O(1);
//   * LTP of the winner (eq.(6)) needs last_pre only in the winner's CTA: the input spike timers are
//     brought up to date lazily there, and nowhere else;
//   * the last winner of each CTA is its *deferred* column: it is LTD-active on every input spike right after
//     its post spike (eq.(7) with small |Dt|) and used to put the longest dependent chain on one warp.  Its LTD
//     events for the next <= nthr raw rows (<= 64 steps) are drawn by the whole CTA at once, and with them its
//     integration sums S(t) = sum_{i active at t} max(q_i - n_i(<t), 0) (n_i(<t): its events on row i at earlier
//     table steps -- decrements clamped at 0 commute), so the owning thread reads S(t) from a table and
//     applies no LTD in the step loop; the events of the committed steps are written back by the CTA when the
//     table is retired (a new winner in the CTA, a rebuild, a window or image boundary).
// Results are bit-identical to the oracle (tests/test_gpu_parity.py runs every case on this kernel and
// on the general one).
#include "snn_internal.h"
#include "snn_device.cuh"

#include <climits>
#include <cstdio>
#include <cstdint>

namespace snn {

// SNN_LEAN_TRACE_CYCLES=1 (compile time) adds the per-section cycle split of the slowest warp to the epoch
// trace (tools/trace_lean.py); off by default, so the step loop carries no clock reads.
#ifndef SNN_LEAN_TRACE_CYCLES
#define SNN_LEAN_TRACE_CYCLES 0
#endif
constexpr bool kTraceCycles = SNN_LEAN_TRACE_CYCLES != 0;

namespace {

template <int BITS, int CPT_> struct LSwar {
  static constexpr int CPT = CPT_;
  static constexpr int CPW = 32 / BITS;
  static constexpr int TPW = CPW / CPT_;
  static constexpr int LW = 32 / CPT_;
  static constexpr uint32_t FM = (1u << BITS) - 1u;
  static constexpr uint32_t LMASK = CPT_ == 1 ? FM : (CPT_ == 2 ? (FM | (FM << 16)) : (FM * 0x01010101u));
  // rows that can be summed into one SWAR word before a lane could overflow (multiple of 4)
  static constexpr int CHUNK = CPT_ == 1 ? (1 << 28) : (int)((((1u << (LW & 31)) - 1u) / FM) & ~3u);
};

constexpr int kDrawRows = 64;        // raw rows one LTD draw covers (two Philox blocks per lane, in flight together)
constexpr int kDefSteps = 64;        // steps one deferred-LTD table covers at most (u64 step masks per input row)
constexpr int kDefMargin = 16;       // a table with fewer steps left than this is rebuilt at the epoch start
constexpr int kDefRowsPerThr = 1;    // raw rows a table draws per thread (an epoch spans ~15 steps of ~6 rows)
constexpr int kSlots = 12;            // fixed row slots per step (steps with more active rows take the general path)
constexpr int kBlk = 2;              // steps one block integrates before running the LIF chains through them

struct LeanLayout {
  size_t slots, wsum, flags, misc, spk, dS, dbits, dev, w, pot, dep, lpre, offs, pst, prow, p8, run, rraw, log, total;
};

__host__ __device__ inline LeanLayout lean_layout(int n_in, int slice_words, int L_pot, int L_dep, int nthr,
                                                  int rows_cap, int offs_cap, int logn) {
  LeanLayout L;
  size_t o = 0;
  L.slots = o; o = align16(o + 2 * kMaxCluster * 2 * 8);     // [parity][rank][2] u64: steps, key
  L.wsum = o;  o = align16(o + 32 * 2 * 8);                  // per warp: steps, key
  L.flags = o; o = align16(o + 4 * 4);                       // early-stop flag per epoch parity
  L.misc = o;  o = align16(o + 40 * 4);
  L.spk = o;   o = align16(o + (size_t)nthr * 4 * 4);                 // LAYER: this CTA's spiking columns
  L.dS = o;    o = align16(o + (size_t)kDefSteps * 4);                // deferred column: S per table step
  L.dbits = o; o = align16(o + (size_t)(kDefRowsPerThr * nthr / 32) * 4);   // deferred column: event bit per raw row
  L.dev = o;   o = align16(o + (size_t)n_in * 8 * 2);                 // deferred column: event steps per input row (x2)
  L.w = o;     o = align16(o + (size_t)slice_words * 4);
  L.pot = o;   o = align16(o + (size_t)(L_pot > 0 ? L_pot : 1) * 4);
  L.dep = o;   o = align16(o + (size_t)(L_dep > 0 ? L_dep : 1) * 4);
  L.lpre = o;  o = align16(o + (size_t)n_in * 4);
  L.offs = o;  o = align16(o + (size_t)(offs_cap + 1) * 4);          // raw row offset of every window step
  L.pst = o;   o = align16(o + (size_t)(offs_cap + 1) * 4);          // padded (x4) start of every window step
  L.prow = o;  o = align16(o + (size_t)(rows_cap + 3 * offs_cap + 4) * 4);   // padded word offsets row*wpr
  L.p8 = o;    o = align16(o + (size_t)(offs_cap + kBlk) * kSlots * 4);   // first kSlots row byte offsets of each step
  L.run = o;   o = align16(o + (size_t)(offs_cap + 1));                   // small steps (<= kSlots rows) from here, <= kBlk
  L.rraw = o;  o = align16(o + (size_t)(rows_cap + kDrawRows) * 4);         // raw rows: step << 16 | row id
  L.log = o;   o = align16(o + (size_t)logn * nthr * 4);
  L.total = o;
  return L;
}

// undo-log entry: rel step (16) | column slot c (2) | applied (1) | row (13)
__device__ __forceinline__ uint32_t lean_log_entry(int rel, int c, bool applied, int row) {
  return ((uint32_t)rel << 16) | ((uint32_t)c << 14) | (applied ? 0x2000u : 0u) | (uint32_t)row;
}

constexpr int kNoStep = 0x7FFFFFFF;

}  // namespace

size_t lean_smem_bytes(int n_in, int slice_words, int L_pot, int L_dep, int nthr, int rows_cap, int offs_cap,
                       int logn) {
  return lean_layout(n_in, slice_words, L_pot, L_dep, nthr, rows_cap, offs_cap, logn).total;
}

// SH: compiled with the cross-rank (column-sharded) exchange; the unsharded instance carries none of it.
// LAY: LAYER WTA (R7) instead of HARD (instantiated unsharded only)
template <int BITS, int CPT_, bool FIXED, bool SH, bool LAY>
__global__ void __launch_bounds__(kEvMaxThreads, 1) present_lean_kernel(const __grid_constant__ LaunchParams lp) {
  using Z = LSwar<BITS, CPT_>;
  constexpr int CPT = Z::CPT;
  constexpr int CPW = Z::CPW;
  constexpr int TPW = Z::TPW;
  constexpr uint32_t FMASK = Z::FM;
  extern __shared__ __align__(16) unsigned char smem[];
  const NetDesc& d0 = lp.descs ? lp.descs[0] : lp.single;
  const int cs = d0.cs;
  const int net = blockIdx.x / cs;
  const int rank = blockIdx.x - net * cs;
  const NetDesc& d = lp.descs ? lp.descs[net] : lp.single;

  const int n_in = d.n_in, n_exc = d.n_exc, qmax = d.q_max, wpr = d.wpr;
  const int T = d.T, flags = d.flags, n_images = d.n_images;
  const int L_pot = d.L_pot, L_dep = d.L_dep, rows_cap = d.rows_cap, offs_cap = d.offs_cap, logn = d.logn;
  const int slice_words = d.slice_words;
  const int nthr = blockDim.x;
  const LeanLayout L = lean_layout(n_in, slice_words, L_pot, L_dep, nthr, rows_cap, offs_cap, logn);
  unsigned long long* s_slots = reinterpret_cast<unsigned long long*>(smem + L.slots);
  unsigned long long* s_wsum = reinterpret_cast<unsigned long long*>(smem + L.wsum);
  int* s_flag = reinterpret_cast<int*>(smem + L.flags);
  int* s_misc = reinterpret_cast<int*>(smem + L.misc);
  uint32_t* s_w = reinterpret_cast<uint32_t*>(smem + L.w);
  uint32_t* s_pot = reinterpret_cast<uint32_t*>(smem + L.pot);
  uint32_t* s_dep = reinterpret_cast<uint32_t*>(smem + L.dep);
  int* s_lpre = reinterpret_cast<int*>(smem + L.lpre);
  uint32_t* s_offs = reinterpret_cast<uint32_t*>(smem + L.offs);
  uint32_t* s_pst = reinterpret_cast<uint32_t*>(smem + L.pst);
  uint32_t* s_prow = reinterpret_cast<uint32_t*>(smem + L.prow);
  uint32_t* s_p8 = reinterpret_cast<uint32_t*>(smem + L.p8);
  uint8_t* s_run = reinterpret_cast<uint8_t*>(smem + L.run);
  uint32_t* s_rraw = reinterpret_cast<uint32_t*>(smem + L.rraw);
  uint32_t* s_log = reinterpret_cast<uint32_t*>(smem + L.log);
  int* s_dS = reinterpret_cast<int*>(smem + L.dS);
  int* s_spk = reinterpret_cast<int*>(smem + L.spk);
  // LAYER WTA (R7): every column that crosses at t* spikes; the summary carries the number of crossers at the
  // earliest step instead of the largest key (HARD)
  constexpr bool layer = LAY;
  uint32_t* s_dbits = reinterpret_cast<uint32_t*>(smem + L.dbits);
  unsigned long long* s_dev = reinterpret_cast<unsigned long long*>(smem + L.dev);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarps = nthr >> 5;
  const int g0 = (rank * d.ngroups) / cs, g1 = ((rank + 1) * d.ngroups) / cs;
  const int col0 = g0 * 32;
  const int cbase = d.col_base;
  const int ncols = min(g1 * 32, n_exc) - col0;
  const int wj = tid / TPW, f = tid % TPW;
  const int fsh = f * BITS;
  const uint32_t* const wcol = s_w + min(wj, wpr - 1);     // threads past the slice read a real word
  int jcol[CPT];                       // local column of slot c (or -1)
  uint32_t valid = 0;
#pragma unroll
  for (int c = 0; c < CPT; ++c) {
    const int jl = wj * CPW + f + TPW * c;
    jcol[c] = (jl < ncols && wj < wpr) ? jl : -1;
    if (jcol[c] >= 0) valid |= 1u << c;
  }
  const uint32_t zero_off = (uint32_t)(n_in * wpr);   // the all-zero row n_in of the slice
  const int nq4 = (n_in + 3) >> 2;

  Lif lif;
  lif.load(d);
  const int vreset = FIXED ? d.Vreset : __float_as_int(d.vresetf);
  const int vinit = FIXED ? d.Vinit : __float_as_int(d.vinitf);
  const int t_ref = d.t_ref, t_inh = d.t_inh;
  const bool keep = (flags & FLAG_KEEP_STATE) != 0;
  const int tbase = keep ? d.t0 : 0;

  // ---- one-time staging
  for (int k = tid; k < L_pot; k += nthr) s_pot[k] = d.pot_m1[k];
  for (int k = tid; k < L_dep; k += nthr) s_dep[k] = d.dep_m1[k];
  {
    const uint4* src = reinterpret_cast<const uint4*>(d.wslices + (size_t)rank * slice_words);
    uint4* dst = reinterpret_cast<uint4*>(s_w);
    for (int k = tid; k < slice_words / 4; k += nthr) dst[k] = src[k];
  }
  if (tid == 0) { s_flag[0] = INT_MAX; s_flag[1] = INT_MAX; }
  for (int i = tid; i < 2 * n_in; i += nthr) s_dev[i] = 0ull;
  // optional per-epoch trace (snn_set_trace; tools/trace_epochs.py): per epoch parity, the latest warp exit
  // (%globaltimer), the longest warp speculation loop (cycles) and the deepest speculation (steps)
  unsigned long long* trace = d.trace ? d.trace + (size_t)rank * d.trace_cap * 8 : nullptr;
  unsigned long long* s_trmax = reinterpret_cast<unsigned long long*>(s_misc + 4);    // [2]
  unsigned long long* s_trloop = reinterpret_cast<unsigned long long*>(s_misc + 8);   // [2]
  int* s_trdepth = s_misc + 12;                                                      // [2]
  unsigned long long* s_trcross = reinterpret_cast<unsigned long long*>(s_misc + 16);  // [2] first crossing (ns)
  if (tid == 0) {
    s_trmax[0] = s_trmax[1] = 0ull; s_trloop[0] = s_trloop[1] = 0ull; s_trdepth[0] = s_trdepth[1] = 0;
    s_trcross[0] = s_trcross[1] = ~0ull;
    for (int q = 24; q < 30; ++q) s_misc[q] = 0;
  }
  int* s_trsteps = s_misc + 24;      // [parity][3]: warp-steps taken by block, general and solo paths (trace)
  unsigned long long tg0 = 0, tg3 = 0, tc3 = 0, tph[5] = {0ull, 0ull, 0ull, 0ull, 0ull};
  int v[CPT], cnt[CPT], lpost[CPT];
#pragma unroll
  for (int c = 0; c < CPT; ++c) {
    v[c] = vinit; cnt[c] = 0; lpost[c] = kNever;
    if (keep && (valid >> c & 1u)) {
      const int jg = col0 + jcol[c];
      v[c] = d.v[jg]; cnt[c] = d.cnt[jg]; lpost[c] = d.last_post[jg];
    }
  }
  if (keep) for (int i = tid; i < n_in; i += nthr) s_lpre[i] = d.last_pre[i];
  uint32_t ltd_trials = 0, ltd_events = 0, ltp_trials = 0, ltp_events = 0;
  unsigned long long act_sum = 0, post_sum = 0;
  uint32_t eng_epochs = 0, eng_hz = 0, eng_resim = 0, eng_spec = 0, eng_undo = 0;
  if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }

  int ep = 0;
  // column sharding: this cluster holds columns [cbase, cbase + n_exc) of a network split over
  // `world` ranks; per epoch the cluster summaries meet in every rank's device mailbox
  const int world = d.world;
  const bool sharded = SH && world > 1;
  const uint32_t seq0 = sharded ? (uint32_t)ld_relaxed_sys_s32(reinterpret_cast<const int*>(&d.mbox->seq)) : 0u;
  if (flags & FLAG_FLOOR) {
    // latency floor probe (SNN_FLOOR_PROBE, bench.py latency_roofline): the same launch shape runs, per image,
    // d.floor_epochs epochs of the synchronisation skeleton alone -- the early-stop signal to every CTA, the
    // warp and CTA summaries, the DSMEM summary stores, the cluster barrier and the decision -- with no
    // integration, LIF or STDP
    unsigned long long chk = 0ull;
    for (int b = 0; b < n_images; ++b) {
      for (int e = 0; e < d.floor_epochs; ++e, ++ep) {
        const int fp = ep & 1;
        const int cst = (rank == (e % cs) && warp == 0) ? e : kNoStep;
        if (rank == (e % cs) && warp == 0 && lane < cs) {
          if (lane == rank) atomicMin(&s_flag[fp], e);
          else red_min_cluster(&s_flag[fp], (uint32_t)lane, e);
        }
        const int wc = __reduce_min_sync(FULL, cst);
        const uint32_t kh = __reduce_max_sync(FULL, (uint32_t)(tid + e));
        if (lane == 0) { s_wsum[2 * warp] = ((unsigned long long)(uint32_t)wc << 32) | (uint32_t)kNoStep; s_wsum[2 * warp + 1] = kh; }
        __syncthreads();
        if (warp == 0) {
          const unsigned long long a = lane < nwarps ? s_wsum[2 * lane] : ~0ull;
          const unsigned long long k = lane < nwarps ? s_wsum[2 * lane + 1] : 0ull;
          const int C = __reduce_min_sync(FULL, (int)(a >> 32));
          const uint32_t K2 = __reduce_max_sync(FULL, (uint32_t)k);
          unsigned long long* slot = s_slots + (size_t)(fp * kMaxCluster + rank) * 2;
          const unsigned long long A = ((unsigned long long)(uint32_t)C << 32) | (uint32_t)kNoStep;
          if (cs == 1) {
            if (lane == 0) { slot[0] = A; slot[1] = K2; }
          } else if (lane < cs) {
            st_cluster_u64(slot, (uint32_t)lane, A);
            st_cluster_u64(slot + 1, (uint32_t)lane, K2);
          }
          if (lane == 0) s_flag[fp ^ 1] = INT_MAX;
        }
        if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }
        const unsigned long long A = lane < cs ? s_slots[(size_t)(fp * kMaxCluster + lane) * 2] : ~0ull;
        const int Pf = __reduce_min_sync(FULL, (int)(A >> 32));
        chk += (unsigned long long)Pf;
      }
      if (rank == 0 && tid == 0 && d.spike_counts) d.spike_counts[b] = 0;
    }
    if (tid == 0 && chk == 0xFFFFFFFFFFFFFFFFull) d.stats[15] = chk;   // keeps the skeleton's results live
    if (cs > 1) { cluster_arrive(); cluster_wait(); }
    return;
  }
  for (int b = 0; b < n_images; ++b) {
    const unsigned long long seed = d.seeds[b];
    if (!keep) {
#pragma unroll
      for (int c = 0; c < CPT; ++c) { v[c] = vinit; cnt[c] = 0; lpost[c] = kNever; }
      for (int i = tid; i < n_in; i += nthr) s_lpre[i] = kNever;
    }
    const uint32_t* offs_g = d.ev_offs + (size_t)b * (T + 1);
    const uint16_t* rows_g = d.ev_rows + (size_t)b * d.rows_stride;
    const bool last_img = (b == n_images - 1);
    const bool rec_out = last_img && d.raster_out != nullptr;
    int img_spikes = 0;
    int ka = 0, kb = 0;            // window steps [ka, kb)
    int lpre_upto = -1;            // s_lpre holds the input spike timers through window step lpre_upto
    int kend_w = 0;                // window end (kb) as seen by the deferred-table helpers
    int k0 = 0;
    // the CTA's deferred column (its last winner, local index Wd; -1 none) and its LTD table: steps [tk0, kcov],
    // raw rows [tr0, tr0 + tnr) of the window; d_lp = its last post spike (absolute step).  CTA-uniform.
    int Wd = -1, d_lp = 0, tk0 = 0, kcov = -1, tr0 = 0, tnr = 0, dbuf = 0;
    bool tvalid = false, pclear = false;
    if (rank == 0 && tid == 0 && T > 0) act_sum += (unsigned long long)(offs_g[T] - offs_g[0]);
    __syncthreads();

    // input spike timers of window steps (lpre_upto, upto]: every CTA thread takes raw rows
    auto lpre_catch_up = [&](int upto) {
      if (upto > lpre_upto) {
        const uint32_t r0 = s_offs[lpre_upto + 1], r1 = s_offs[upto + 1];
        for (uint32_t r = r0 + tid; r < r1; r += nthr) {
          const uint32_t rr = s_rraw[r];
          atomicMax(&s_lpre[rr & 0xFFFFu], tbase + ka + (int)(rr >> 16));
        }
        lpre_upto = upto;
      }
    };

    // ---- deferred column (CTA-cooperative; every thread calls these at the same point, arguments CTA-uniform).
    // The per-row event masks are double-buffered (s_dev + dbuf * n_in), so clearing a retired table's masks and
    // drawing the next table share one barrier phase.  Phases: apply | clear + draw | sums.
    // apply: write back the table's eq.(7) events of the steps <= kc (decrements of one row clamp at 0, so their
    // total is applied at once by the thread holding the row's first event), count them and their trials (R20)
    auto dtab_apply = [&](int kc) {
      const unsigned long long* dev = s_dev + dbuf * n_in;
      const int ww = Wd / CPW, wsh = (Wd % CPW) * BITS;
      const int relc = kc - tk0;
      for (int r = tid; r < tnr; r += nthr) {
        const uint32_t rr = s_rraw[tr0 + r];
        const int k = ka + (int)(rr >> 16);
        if (k > kc) continue;
        const int i = (int)(rr & 0xFFFFu);
        if (tbase + k - d_lp < L_dep) ++ltd_trials;
        if (!((s_dbits[r >> 5] >> (r & 31)) & 1u)) continue;
        ++ltd_events;
        const unsigned long long m = dev[i];
        if (__popcll(m & ((1ull << (k - tk0)) - 1ull)) != 0) continue;    // not the row's first event
        const int n = __popcll(relc >= 63 ? m : (m & ((2ull << relc) - 1ull)));
        // the column's field of row i is this thread's alone (other fields may be in an undo: atomic)
        uint32_t* pw = s_w + i * wpr + ww;
        const int dec = min(n, (int)((*pw >> wsh) & FMASK));
        if (dec) atomicSub(pw, (uint32_t)dec << wsh);
      }
      tvalid = false;
      pclear = true;                                   // its masks are cleared in the next phase
    };
    auto dtab_clear = [&]() {
      if (!pclear) return;
      unsigned long long* dev = s_dev + dbuf * n_in;
      for (int r = tid; r < tnr; r += nthr) dev[s_rraw[tr0 + r] & 0xFFFFu] = 0ull;
      pclear = false;
    };
    // draw: the next table from window step k_start (the column's codes are committed through k_start - 1 by the
    // end of this phase): eq.(7) draws of the column for the next <= kDefRowsPerThr*nthr raw rows (whole steps, <= kDefSteps
    // of them), one row per thread and iteration, into the other mask buffer.  Returns false (no table) when the
    // column is no longer LTD-active or the next step alone has more rows than a table covers.
    int nt_r0 = 0, nt_nr = 0, nt_kc = -1;
    auto dtab_draw = [&](int k_start) -> bool {
      if (tbase + k_start - d_lp >= L_dep) { Wd = -1; return false; }   // no longer LTD-active (R10)
      const int r0 = (int)s_offs[k_start - ka];
      const int nrw = (int)s_offs[kend_w - ka];
      int kc = kend_w - 1;
      if (r0 + kDefRowsPerThr * nthr < nrw) kc = ka + (int)(s_rraw[r0 + kDefRowsPerThr * nthr] >> 16) - 1;
      kc = min(kc, k_start + kDefSteps - 1);
      if (kc < k_start) return false;                  // a step of more rows than a table: the column stays in the loop
      const int nr = (int)s_offs[kc + 1 - ka] - r0;
      const int Wg = cbase + col0 + Wd;
      unsigned long long* dev = s_dev + (dbuf ^ 1) * n_in;
      for (int k = tid; k < kDefSteps; k += nthr) s_dS[k] = 0;
      bool ev[kDefRowsPerThr];
#pragma unroll
      for (int it = 0; it < kDefRowsPerThr; ++it) {
        const int r = it * nthr + tid;
        ev[it] = false;
        if (r < nr) {
          const uint32_t rr = s_rraw[r0 + r];
          const int k = ka + (int)(rr >> 16);
          const int t = tbase + k;
          const int D = t - d_lp;                                            // R10: Dt = -D < 0
          if (D < L_dep) {
            const uint4 u = philox((uint32_t)t, rr & 0xFFFFu, (uint32_t)(Wg >> 2), TAG_LTD, seed);   // eq.(7), R13
            ev[it] = pick(u, Wg & 3) <= s_dep[D];
          }
          if (ev[it]) atomicOr(&dev[rr & 0xFFFFu], 1ull << (k - k_start));
        }
      }
#pragma unroll
      for (int it = 0; it < kDefRowsPerThr; ++it) {
        const uint32_t m = __ballot_sync(FULL, ev[it]);
        if (lane == 0) s_dbits[it * nwarps + warp] = m;
      }
      nt_r0 = r0; nt_nr = nr; nt_kc = kc;
      tk0 = k_start;
      return true;
    };
    // sums (after a barrier): S(t) of every table step from the clamped codes; the table goes live
    auto dtab_sums = [&]() {
      dbuf ^= 1;
      const unsigned long long* dev = s_dev + dbuf * n_in;
      const int ww = Wd / CPW, wsh = (Wd % CPW) * BITS;
      for (int r = tid; r < nt_nr; r += nthr) {
        const uint32_t rr = s_rraw[nt_r0 + r];
        const int rel = ka + (int)(rr >> 16) - tk0;
        const int i = (int)(rr & 0xFFFFu);
        const int n = __popcll(dev[i] & ((1ull << rel) - 1ull));            // earlier events on the row
        const int q = (int)((s_w[i * wpr + ww] >> wsh) & FMASK);
        if (q > n) atomicAdd(&s_dS[rel], q - n);                           // eq.(3) with the clamped codes
      }
      kcov = nt_kc; tr0 = nt_r0; tnr = nt_nr; tvalid = true;
    };
    // retire the table completely (window / image end)
    auto dtab_retire = [&](int kc) {
      dtab_apply(kc);
      __syncthreads();
      dtab_clear();
      __syncthreads();
    };
    // (re)build from k_start, retiring the current table (if any) through k_start - 1
    auto dtab_rebuild = [&](int k_start) {
      if (tvalid) { dtab_apply(k_start - 1); __syncthreads(); }
      dtab_clear();
      const bool ok = dtab_draw(k_start);
      __syncthreads();
      if (ok) { dtab_sums(); __syncthreads(); }
    };

    while (k0 < T) {
      // ---------------------------------------------------------- stage the active-row window
      if (k0 >= kb) {
        if (tvalid) dtab_retire(min(k0 - 1, kcov));                 // the table indexes the old window
        else if (pclear) { dtab_clear(); __syncthreads(); }
        __syncthreads();
        if (kb > ka) lpre_catch_up(kb - 1 - ka);                   // finish the old window's timers
        __syncthreads();
        ka = k0;
        lpre_upto = -1;
        const int n_o = min(offs_cap, T - ka);
        const uint32_t wbase = offs_g[ka];
        for (int x = tid; x <= n_o; x += nthr) s_offs[x] = offs_g[ka + x] - wbase;
        if (tid == 0) s_misc[0] = 0;
        __syncthreads();
        int fit = 0;
        for (int x = tid + 1; x <= n_o; x += nthr) {
          const uint32_t padded = s_offs[x] + 3u * (uint32_t)x;      // upper bound of the padded length
          fit += (s_offs[x] <= (uint32_t)rows_cap && padded <= (uint32_t)(rows_cap + 3 * offs_cap)) ? 1 : 0;
        }
        if (fit) atomicAdd(&s_misc[0], fit);
        __syncthreads();
        const int nsteps = max(1, s_misc[0]);    // rows_cap >= n_in: one step always fits
        kb = ka + nsteps;
        // padded starts: warp 0 scans the per-step group counts
        if (warp == 0) {
          const int per = (nsteps + 31) / 32;
          const int lo = min(nsteps, lane * per), hi = min(nsteps, lo + per);
          uint32_t sum = 0;
          for (int x = lo; x < hi; ++x) sum += (s_offs[x + 1] - s_offs[x] + 3u) & ~3u;
          uint32_t incl = sum;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
          }
          uint32_t run = incl - sum;
          for (int x = lo; x < hi; ++x) { s_pst[x] = run; run += (s_offs[x + 1] - s_offs[x] + 3u) & ~3u; }
          if (lane == 31) s_pst[nsteps] = incl;
        }
        __syncthreads();
        // raw rows (step << 16 | id) and padded word offsets; one thread per step
        const uint32_t nrows = s_offs[nsteps];
        for (int x = tid; x < nsteps; x += nthr) {
          const uint32_t o0 = s_offs[x], o1 = s_offs[x + 1], p0 = s_pst[x], p1 = s_pst[x + 1];
          for (uint32_t r = o0; r < o1; ++r) {
            const uint32_t i = rows_g[wbase + r];
            s_rraw[r] = ((uint32_t)x << 16) | i;
            s_prow[p0 + (r - o0)] = i * (uint32_t)wpr;
          }
          for (uint32_t q = p0 + (o1 - o0); q < p1; ++q) s_prow[q] = zero_off;
#pragma unroll
          for (int j = 0; j < kSlots; ++j) s_p8[kSlots * x + j] = 4u * ((uint32_t)j < o1 - o0 ? s_prow[p0 + j] : zero_off);
        }
        for (int x = nsteps * kSlots + tid; x < (nsteps + kBlk) * kSlots; x += nthr) s_p8[x] = 4u * zero_off;
        for (int x = tid; x < kDrawRows; x += nthr) s_rraw[nrows + x] = 0xFFFF0000u;   // draw pads (never an event)
        for (int x = tid; x < nsteps; x += nthr) {
          int run = 0;
          while (run < kBlk && x + run < nsteps && s_offs[x + run + 1] - s_offs[x + run] <= (uint32_t)kSlots) ++run;
          s_run[x] = (uint8_t)run;
        }
        __syncthreads();
      }
      kend_w = kb;
      // (re)build the deferred column's table when it is missing or covers too little of this epoch
      if (Wd >= 0 && (!tvalid || kcov < min(k0 + kDefMargin, kb - 1))) {
        dtab_rebuild(k0);
      }
      const int kend = kb;
      const int fp = ep & 1;
      const uint32_t flag_addr = smem_u32(&s_flag[fp]);
      const long long tl0 = trace ? clock64() : 0ll;
      // trace (SNN_LEAN_TRACE_CYCLES builds): cycles of the warp in held runs, block steps, general steps
      long long c_held = 0, c_blk = 0, c_gen = 0, t_it = 0;
#define LEAN_CYC(acc) do { if (kTraceCycles && trace) (acc) += clock64() - t_it; } while (0)
      if (trace && tid == 0) tg0 = globaltimer();

      // ---------------------------------------------------------- speculation (warp-synchronous)
      int cnt0[CPT], v1[CPT], cnt1[CPT];
#pragma unroll
      for (int c = 0; c < CPT; ++c) { cnt0[c] = cnt[c]; v1[c] = v[c]; cnt1[c] = cnt[c]; }
      // the deferred column (this thread's slot dslot, if any) takes S from its table and no in-loop LTD
      int dslot = -1;
#pragma unroll
      for (int c = 0; c < CPT; ++c)
        if (tvalid && (valid >> c & 1u) && jcol[c] == Wd) dslot = c;
      // its warp stops before the first step the table does not cover (the epoch then ends there, no spike)
      const bool wdef = __any_sync(FULL, dslot >= 0);
      const int kstop = wdef ? kcov + 1 : kend;
      uint32_t dmask = 0;                                  // LTD-active columns of this thread (R10)
#pragma unroll
      for (int c = 0; c < CPT; ++c)
        if ((valid >> c & 1u) && c != dslot && lpost[c] >= 0 && (tbase + k0 - lpost[c]) < L_dep) dmask |= 1u << c;
      const uint32_t wdirty = __ballot_sync(FULL, dmask != 0);
      // A packed word belongs to TPW consecutive lanes of one warp and, during speculation, only LTD writes
      // codes (each lane its own fields).  When no two LTD-active lanes share a word, a lane's decrement is
      // the only write to that word: a plain read-modify-write replaces the shared-memory atomic (-7 % time).
      const uint32_t same_word = (TPW >= 32 ? FULL : ((1u << TPW) - 1u)) << (TPW >= 32 ? 0 : (lane & ~(TPW - 1)));
      const bool ltd_plain = !__any_sync(FULL, dmask != 0 && __popc(same_word & wdirty) > 1);
      // countdowns only run down during speculation (R6, R7), so the warp's first step with a live column is
      // k0 + the smallest countdown of its valid columns (no per-step vote needed)
      // the deferred column runs ahead on its own (below); the step loop handles the other columns (lvalid)
      const uint32_t lvalid = valid & ~(dslot >= 0 ? (1u << dslot) : 0u);
      int live_from;
      {
        int mnd = INT_MAX;
#pragma unroll
        for (int c = 0; c < CPT; ++c)
          if (lvalid >> c & 1u) mnd = min(mnd, cnt[c]);
        mnd = __reduce_min_sync(FULL, mnd);
        live_from = mnd == INT_MAX ? INT_MAX : k0 + mnd;
      }
      int kk = k0;
      int p_done = k0 - 1;           // last step fully processed by this thread
      int cstep = kNoStep;           // crossing step (the warp stops right after it)
      int hstep = kNoStep;           // undo log full: stopped before this step
      unsigned long long ckey = 0ull;    // HARD: best WTA key at cstep; LAYER: number of own columns crossing at cstep
      uint32_t cmk = 0u;                 // own columns crossing at cstep
      int nlog = 0;
      int dr0 = INT_MIN;             // warp-uniform raw start of the drawn LTD row range [dr0, dr0 + kDrawRows)
      unsigned long long evm[CPT];   // LTD event bits of raw rows [dr0, dr0 + 64) (owning lane)
#pragma unroll
      for (int c = 0; c < CPT; ++c) evm[c] = 0ull;
      // event bits of column slot c for raw rows [a0, a1) (a1 - a0 <= 32, inside the drawn range)
      auto evbits = [&](int c, int a0, int a1) -> uint32_t {
        const int nr = a1 - a0;
        return nr <= 0 ? 0u : ((uint32_t)(evm[c] >> (a0 - dr0)) & (nr >= 32 ? FULL : ((1u << nr) - 1u)));
      };

      // a crossing at window step kc: lower the early-stop flag of every CTA of the cluster (lane r -> CTA r)
      const uint32_t cur = seq0 + (uint32_t)ep + 1u;        // shard-exchange epoch number (never 0 in use)
      auto signal_cross = [&](int kc) {
        if (trace && lane == 0) atomicMin(&s_trcross[fp], globaltimer());
        if (lane < cs) {
          if (lane == rank) atomicMin(&s_flag[fp], kc);
          else red_min_cluster(&s_flag[fp], (uint32_t)lane, kc);
        }
        if (sharded && lane < world && lane != d.shard)      // lane r -> rank r (NVLink peer reduction)
          red_max_sys_u64(&d.peers[lane]->flag, ((unsigned long long)cur << 32) | (0xFFFFFFFFu - (uint32_t)kc));
      };

      // LTD draws of every (lane, column) pair of the warp for raw rows [base, base + 64): lanes over rows,
      // two rows per lane whose Philox blocks are independent (one chain's latency for 64 rows)
      auto draw = [&](int base) {
        const uint32_t rr0 = s_rraw[base + lane], rr1 = s_rraw[base + 32 + lane];
        const int nrw = (int)s_offs[kend - ka];
        const int t0 = tbase + ka + (int)(rr0 >> 16), t1 = tbase + ka + (int)(rr1 >> 16);
        const uint32_t i0 = rr0 & 0xFFFFu, i1 = rr1 & 0xFFFFu;
        const bool ok0 = (rr0 >> 16) != 0xFFFFu && base + lane < nrw;
        const bool ok1 = (rr1 >> 16) != 0xFFFFu && base + 32 + lane < nrw;
#pragma unroll 1
        for (uint32_t lm = wdirty; lm; lm &= lm - 1) {
          const int Ls = __ffs(lm) - 1;
          const uint32_t dm = __shfl_sync(FULL, dmask, Ls);
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            if (!(dm >> c & 1u)) continue;                 // warp-uniform
            const int jl = __shfl_sync(FULL, jcol[c], Ls);
            const int lp = __shfl_sync(FULL, lpost[c], Ls);
            const int jg = cbase + col0 + jl;
            const int D0 = t0 - lp, D1 = t1 - lp;
            const uint4 u0 = philox((uint32_t)t0, i0, (uint32_t)(jg >> 2), TAG_LTD, seed);   // eq.(7), R13
            const uint4 u1 = philox((uint32_t)t1, i1, (uint32_t)(jg >> 2), TAG_LTD, seed);
            const bool in0 = ok0 && D0 < L_dep, in1 = ok1 && D1 < L_dep;
            const bool bit0 = in0 && pick(u0, jg & 3) <= s_dep[in0 ? D0 : 0];
            const bool bit1 = in1 && pick(u1, jg & 3) <= s_dep[in1 ? D1 : 0];
            const uint32_t m0 = __ballot_sync(FULL, bit0), m1 = __ballot_sync(FULL, bit1);
            if (lane == Ls) evm[c] = ((unsigned long long)m1 << 32) | m0;
          }
        }
      };

      // LTD events of one step (rows [a0, a1) within the drawn window, <= 32 rows), applied in row order;
      // events of steps after k0 are logged for a possible rollback (R14: old last_post, eq.(7))
      auto ltd_apply = [&](int kstep, int a0, int a1) {
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
          if (!(dmask >> c & 1u)) continue;
          uint32_t em = evbits(c, a0, a1);
          const int shc = fsh + c * Z::LW;
          if (ltd_plain) {                             // warp-uniform: this lane is the only writer of its words
            while (em) {
              const int xr = __ffs(em) - 1;
              em &= em - 1;
              const int i = (int)(s_rraw[a0 + xr] & 0xFFFFu);
              uint32_t* pw = s_w + i * wpr + wj;
              const uint32_t wv = *pw;
              const bool applied = ((wv >> shc) & FMASK) != 0u;
              if (applied) *pw = wv - (1u << shc);
              ++ltd_events;
              if (kstep > k0) s_log[nlog++ * nthr + tid] = lean_log_entry(kstep - k0, c, applied, i);
            }
          } else {                                     // another LTD-active lane shares a word: atomics
            while (em) {
              const int xr = __ffs(em) - 1;
              em &= em - 1;
              const int i = (int)(s_rraw[a0 + xr] & 0xFFFFu);
              uint32_t* pw = s_w + i * wpr + wj;
              const bool applied = ((*pw >> shc) & FMASK) != 0u;
              if (applied) atomicSub(pw, 1u << shc);
              ++ltd_events;
              if (kstep > k0) s_log[nlog++ * nthr + tid] = lean_log_entry(kstep - k0, c, applied, i);
            }
          }
        }
      };

      // ---- the deferred column runs ahead alone: its S(t) comes from the table and it has no in-loop LTD, so its
      // lane walks its eqs.(1)(2) chain to its first crossing (or the table's end, or a crossing already reported)
      // at once and lowers the early-stop flag; the step loop below then handles only the warp's other columns.
      // Past t* nothing it computed is kept (RESET: every column restarts from its countdown), so running ahead
      // is exact; for a replay (no spike) it leaves its state after step k0 in v1/cnt1 like every column.
      int p_look = k0 - 1;
      if (wdef) {                                                  // warp-uniform
        int cd = kNoStep, last = k0 - 1;
        unsigned long long keyd = 0ull;
        const int fl0 = ld_volatile_shared_u32addr(flag_addr);
        const int lim = fl0 == INT_MAX ? kstop : min(kstop, fl0 + 1);
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
          if (c != dslot) continue;
          int m = k0;
          const int nh = min(cnt[c], max(lim - k0, 0));          // held steps: the countdown runs down (R6, R7)
          cnt[c] -= nh;
          m += nh;
          if (nh > 0) { v1[c] = v[c]; cnt1[c] = cnt0[c] - 1; }   // state after step k0 (held at k0)
          for (; m < lim; ++m) {
            const bool cr = lif.post_t<FIXED>(v[c], lif.pre_t<FIXED>(s_dS[m - tk0]));   // eqs.(1)(2), eq.(3) from the table
            if (m == k0) { v1[c] = v[c]; cnt1[c] = 0; }
            if (cr) {
              cd = m;
              keyd = ((unsigned long long)lif.ord(v[c]) << 32) | (0xFFFFFFFFu - (uint32_t)(cbase + col0 + jcol[c]));
              break;
            }
          }
          last = cd != kNoStep ? cd : m - 1;
        }
        const int dl = __ffs(__ballot_sync(FULL, dslot >= 0)) - 1;
        const int cdw = __shfl_sync(FULL, cd, dl);
        const int lastw = __shfl_sync(FULL, last, dl);
        if (dslot >= 0) {
          p_look = last;
          if (cd != kNoStep) { cstep = cd; ckey = layer ? 1ull : keyd; cmk = 1u << dslot; }
        }
        if (cdw != kNoStep) {
          signal_cross(cdw);
        } else if (lastw == kstop - 1 && kstop < kend) {          // the table ends first: the epoch ends there
          if (dslot >= 0) hstep = kstop;
          signal_cross(kstop - 1);
        }
      }
#ifdef SNN_LEAN_DEBUG
      long long dbg_it = 0;
#endif
      while (true) {
#ifdef SNN_LEAN_DEBUG
        if (++dbg_it > 20000) {
          if (lane == 0) printf("SPIN rank %d warp %d k0 %d kk %d kend %d flag %d\n", rank, warp, k0, kk, kend,
                                ld_volatile_shared_u32addr(flag_addr));
          __trap();
        }
#endif
        // one lane's read of the early-stop flag decides for the warp (lanes that executed the load apart
        // could otherwise see different values and leave the loop apart); read fresh every iteration: an
        // iteration may be a block of steps, so a stale value would let the warp overrun t* by a whole block
        if (sharded && lane == 0) {        // the other ranks' early-stop signals for this epoch
          const unsigned long long gf = ld_relaxed_sys_u64(&d.mbox->flag);
          if ((uint32_t)(gf >> 32) == cur) atomicMin(&s_flag[fp], (int)(0xFFFFFFFFu - (uint32_t)gf));
        }
        const int fl = __shfl_sync(FULL, ld_volatile_shared_u32addr(flag_addr), 0);
        if (kk >= kstop || kk > fl) break;                       // warp-uniform
        if (kTraceCycles && trace) t_it = clock64();
        const int x = kk - ka;
        const int o0 = (int)s_offs[x], o1 = (int)s_offs[x + 1];
        const int ps = (int)s_pst[x], pe = (int)s_pst[x + 1];   // padded row range (integration below)
        const bool wlive = kk >= live_from;                      // warp-uniform
        if (!wlive) {                                            // held warp: skip the run
          int n = min(live_from - kk, kstop - kk);
          if (fl != INT_MAX) n = min(n, fl - kk + 1);
          bool stop = false;
          if (wdirty) {
            // LTD-active warp: nothing integrates during the run, so only its LTD events (in step order)
            // remain -- applied here without the per-step machinery; a step of > 32 rows ends the run
            // (the general path handles it), a full undo log stops the speculation before that step
            const long long tq = (kTraceCycles && trace) ? clock64() : 0ll;
            int m = 0;
            for (; m < n; ++m) {
              const int xs = kk + m - ka;
              const int a0 = (int)s_offs[xs], a1 = (int)s_offs[xs + 1];
              if (a1 - a0 > 32) break;                                               // warp-uniform
              if (a0 < dr0 || a1 > dr0 + kDrawRows) {
                const long long td = (kTraceCycles && trace) ? clock64() : 0ll;
                draw(a0);
                dr0 = a0;
                (void)td;
              }
              int nev = 0;
#pragma unroll
              for (int c = 0; c < CPT; ++c) nev += __popc(evbits(c, a0, a1));
              const bool full = (kk + m) > k0 && nlog + nev > logn;
              if (__any_sync(FULL, full)) {
                if (full) hstep = kk + m;
                stop = true;
                break;
              }
              if (nev) ltd_apply(kk + m, a0, a1);                    // this lane has events in the step
            }
            n = m;
            (void)tq;
          }
          if (n == 0 && !stop) goto general_step;                                  // a big step first
          if (n > 0 && kk == k0) {
#pragma unroll
            for (int c = 0; c < CPT; ++c) if (lvalid >> c & 1u) { v1[c] = v[c]; cnt1[c] = cnt[c] - 1; }
          }
#pragma unroll
          for (int c = 0; c < CPT; ++c) if (lvalid >> c & 1u) cnt[c] -= n;
          kk += n;
          p_done = kk - 1;
          LEAN_CYC(c_held);
          if (stop) break;
          continue;
        }
        if (!wdirty && kk > k0) {                                // warp-uniform
          // a block of up to kBlk steps of <= kSlots rows: every sum first (independent loads), then the
          // eqs.(1)(2) chains through them; a crossing ends the block (the sums after it are discarded)
          int nbs = min((int)s_run[x], kstop - kk);
          if (fl != INT_MAX) nbs = min(nbs, fl - kk + 1);
          if (nbs > 0) {
            // sums of the block's steps and the v-independent part of eq.(1) (ahead of the chains); every step of the
            // block is summed unconditionally (branch-free, so all loads are in flight together; s_p8 is padded with
            // the zero row past the window), sums past nbs are discarded
            const char* const wb = reinterpret_cast<const char*>(wcol);
            auto ldw = [&](uint32_t off) { return (*reinterpret_cast<const uint32_t*>(wb + off) >> fsh) & Z::LMASK; };
            uint32_t acc[kBlk];
#pragma unroll
            for (int j = 0; j < kBlk; ++j) {
              uint32_t a4[kSlots / 4];
#pragma unroll
              for (int g = 0; g < kSlots / 4; ++g) {
                const uint4 m = *reinterpret_cast<const uint4*>(s_p8 + kSlots * (x + j) + 4 * g);
                a4[g] = (ldw(m.x) + ldw(m.y)) + (ldw(m.z) + ldw(m.w));
              }
              uint32_t a = a4[0];
#pragma unroll
              for (int g = 1; g < kSlots / 4; ++g) a += a4[g];
              acc[j] = a;
            }
            int yv[kBlk][CPT];
#pragma unroll
            for (int j = 0; j < kBlk; ++j) {
              const int Sd = (dslot >= 0 && j < nbs) ? s_dS[kk + j - tk0] : 0;
#pragma unroll
              for (int c = 0; c < CPT; ++c) {
                const int Sc = c == dslot ? Sd
                                          : (int)(Z::LW == 32 ? acc[j] : ((acc[j] >> (c * Z::LW)) & ((1u << (Z::LW & 31)) - 1u)));
                yv[j][c] = lif.pre_t<FIXED>(Sc);
              }
            }
            // the chains: eqs.(1)(2) step by step; a crossing ends the block (the sums after it are discarded)
            uint32_t cmb = 0;
            int jb = 0;
#pragma unroll
            for (int j = 0; j < kBlk; ++j) {
              if (j >= nbs || cmb) continue;                     // warp-uniform
              jb = j;
              uint32_t cm = 0;
#pragma unroll
              for (int c = 0; c < CPT; ++c) {
                if (!(lvalid >> c & 1u)) continue;
                if (cnt[c] > 0) { --cnt[c]; continue; }             // refractory / inhibited: hold v (R6, R7)
                if (lif.post_t<FIXED>(v[c], yv[j][c])) cm |= 1u << c;   // eq.(2): v > v_th
              }
              if (cm) {
                // (the thread's deferred column may have reported a LATER crossing in its run ahead: an earlier
                // one replaces its key, an equal one competes with it)
                if (kk + j < cstep) { cstep = kk + j; ckey = 0ull; cmk = 0u; }
                cmk |= cm;
                if (layer) {
                  ckey += (unsigned long long)__popc(cm);
                } else {
#pragma unroll
                  for (int c = 0; c < CPT; ++c) {
                    if (!(cm >> c & 1u)) continue;
                    const unsigned long long key = ((unsigned long long)lif.ord(v[c]) << 32) |
                                                   (0xFFFFFFFFu - (uint32_t)(cbase + col0 + jcol[c]));
                    ckey = key > ckey ? key : ckey;
                  }
                }
              }
              cmb = __any_sync(FULL, cm != 0) ? 1u : 0u;
            }
            LEAN_CYC(c_blk);
            if (trace && lane == 0) atomicAdd(&s_trsteps[fp * 3 + 0], cmb ? jb + 1 : nbs);
            if (cmb) {
              p_done = kk + jb;
              signal_cross(kk + jb);
              break;
            }
            kk += nbs;
            p_done = kk - 1;
            continue;
          }
        }
      general_step:
        // ---- this step's LTD events of the warp's LTD-active pairs (draws cover 32 rows ahead)
        const bool big = (o1 - o0) > 32;
        int nev = 0;
        if (wdirty) {
          if (!big && (o0 < dr0 || o1 > dr0 + kDrawRows)) {
            const long long tq = (kTraceCycles && trace) ? clock64() : 0ll;
            draw(o0);
            dr0 = o0;
            (void)tq;
          }
          if (!big) {
#pragma unroll
            for (int c = 0; c < CPT; ++c) nev += __popc(evbits(c, o0, o1));
          } else {
            nev = __popc(dmask) * (o1 - o0);                     // conservative bound (steps of > 32 rows)
          }
          // undo-log space for this step (steps after k0 are logged); else stop before it
          const bool full = kk > k0 && nlog + nev > logn;
          if (__any_sync(FULL, full)) {
            if (full) hstep = kk;
            break;
          }
        }
        // ---- (a2) eq.(3) + (a3) eqs.(1)(2): integrate the step's rows, Euler step of live columns
        uint32_t cm = 0;
        const long long tq_int = (kTraceCycles && trace) ? clock64() : 0ll;
        if (wlive) {
          int S[CPT];
#pragma unroll
          for (int c = 0; c < CPT; ++c) S[c] = 0;
          int q = ps;
          while (q < pe) {
            const int qe = min(pe, q + Z::CHUNK);
            uint32_t acc = 0u;
            for (; q + 4 < qe; q += 8) {         // two padded groups per trip: both offset loads in flight
              const uint4 m = *reinterpret_cast<const uint4*>(s_prow + q);
              const uint4 m2 = *reinterpret_cast<const uint4*>(s_prow + q + 4);
              acc += ((wcol[m.x] >> fsh) & Z::LMASK) + ((wcol[m.y] >> fsh) & Z::LMASK) +
                     ((wcol[m.z] >> fsh) & Z::LMASK) + ((wcol[m.w] >> fsh) & Z::LMASK);
              acc += ((wcol[m2.x] >> fsh) & Z::LMASK) + ((wcol[m2.y] >> fsh) & Z::LMASK) +
                     ((wcol[m2.z] >> fsh) & Z::LMASK) + ((wcol[m2.w] >> fsh) & Z::LMASK);
            }
            if (q < qe) {
              const uint4 m = *reinterpret_cast<const uint4*>(s_prow + q);
              acc += ((wcol[m.x] >> fsh) & Z::LMASK) + ((wcol[m.y] >> fsh) & Z::LMASK) +
                     ((wcol[m.z] >> fsh) & Z::LMASK) + ((wcol[m.w] >> fsh) & Z::LMASK);
              q += 4;
            }
#pragma unroll
            for (int c = 0; c < CPT; ++c)
              S[c] += (int)(Z::LW == 32 ? acc : ((acc >> (c * Z::LW)) & ((1u << (Z::LW & 31)) - 1u)));
          }
          if (dslot >= 0) {                                         // the deferred column: S from its table
            const int Sd = s_dS[kk - tk0];
#pragma unroll
            for (int c = 0; c < CPT; ++c) if (c == dslot) S[c] = Sd;
          }
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            if (!(lvalid >> c & 1u)) continue;
            if (cnt[c] > 0) { --cnt[c]; continue; }                 // refractory / inhibited: hold v (R6, R7)
            if (lif.step_t<FIXED>(v[c], S[c])) cm |= 1u << c;       // eq.(2): v > v_th
          }
        } else {
#pragma unroll
          for (int c = 0; c < CPT; ++c) if ((lvalid >> c & 1u) && cnt[c] > 0) --cnt[c];
        }
        (void)tq_int;
        const long long tq_ev = (kTraceCycles && trace) ? clock64() : 0ll;
        // ---- (a5) LTD events of the step (old last_post, R14), applied in step order
        if (wdirty && dmask) {
          const int t = tbase + kk;
          if (!big) {
            if (nev) ltd_apply(kk, o0, o1);                      // this lane has events in the step
          } else {
            // steps with more than 32 active rows: the lane draws its own rows serially (rare)
#pragma unroll
            for (int c = 0; c < CPT; ++c) {
              if (!(dmask >> c & 1u)) continue;
              const int D = t - lpost[c];
              if (D >= L_dep) continue;
              const uint32_t thr = s_dep[D];
              const int jg = cbase + col0 + jcol[c];
              const int shc = fsh + c * Z::LW;
              for (int r = o0; r < o1; ++r) {
                const int i = (int)(s_rraw[r] & 0xFFFFu);
                const uint4 u = philox((uint32_t)t, (uint32_t)i, (uint32_t)(jg >> 2), TAG_LTD, seed);
                if (pick(u, jg & 3) <= thr) {
                  uint32_t* pw = s_w + i * wpr + wj;
                  const bool applied = ((*pw >> shc) & FMASK) != 0u;
                  if (applied) atomicSub(pw, 1u << shc);
                  ++ltd_events;
                  if (kk > k0) s_log[nlog++ * nthr + tid] = lean_log_entry(kk - k0, c, applied, i);
                }
              }
            }
          }
        }
        (void)tq_ev;
        if (kk == k0) {
#pragma unroll
          for (int c = 0; c < CPT; ++c) if (lvalid >> c & 1u) { v1[c] = v[c]; cnt1[c] = cnt[c]; }
        }
        p_done = kk;
        if (cm) {                                                // crossing: the WTA key (R7)
          if (kk < cstep) { cstep = kk; ckey = 0ull; cmk = 0u; }   // (see the block path)
          cmk |= cm;
          if (layer) {
            ckey += (unsigned long long)__popc(cm);
          } else {
#pragma unroll
            for (int c = 0; c < CPT; ++c) {
              if (!(cm >> c & 1u)) continue;
              const unsigned long long key = ((unsigned long long)lif.ord(v[c]) << 32) |
                                             (0xFFFFFFFFu - (uint32_t)(cbase + col0 + jcol[c]));
              ckey = key > ckey ? key : ckey;
            }
          }
        }
        LEAN_CYC(c_gen);
        if (trace && lane == 0) atomicAdd(&s_trsteps[fp * 3 + 1], 1);
        if (__any_sync(FULL, cm != 0)) { signal_cross(kk); break; }
        ++kk;
      }
      {                                                          // tell the cluster (and the ranks) where to stop
        const int hw = __reduce_min_sync(FULL, hstep);
        if (hstep != kNoStep) ++eng_hz;
        if (hw != kNoStep) signal_cross(hw - 1);
      }
      p_done = max(p_done, p_look);
      if (valid) eng_spec += (uint32_t)(p_done - k0 + 1) * (uint32_t)__popc(valid);
      if (trace && lane == 0) {
        atomicMax(&s_trmax[fp], globaltimer());
        const unsigned long long f16 = 0xFFFFull;
        const unsigned long long loop16 = min((unsigned long long)(clock64() - tl0) >> 4, f16);
        atomicMax(&s_trloop[fp], (loop16 << 48) | (min((unsigned long long)c_held >> 4, f16) << 32) |
                                 (min((unsigned long long)c_blk >> 4, f16) << 16) | min((unsigned long long)c_gen >> 4, f16));
        atomicMax(&s_trdepth[fp], p_done - k0 + 1);
      }

      // ---------------------------------------------------------- CTA summary -> cluster exchange
#ifdef SNN_LEAN_DEBUG
      if (lane == 0 && k0 >= 116) printf("SPEC r %d w %d k0 %d kk %d p_done %d cstep %d hstep %d\n", rank, warp, k0, kk, p_done, cstep, hstep);
#endif
      {
        const int wc = __reduce_min_sync(FULL, cstep);
        const int wh = __reduce_min_sync(FULL, hstep);
        const uint32_t kh = __reduce_max_sync(FULL, cstep == wc ? (uint32_t)(ckey >> 32) : 0u);
        const uint32_t kl = layer ? __reduce_add_sync(FULL, cstep == wc ? (uint32_t)ckey : 0u)   // LAYER: count
                                  : __reduce_max_sync(FULL, (cstep == wc && (uint32_t)(ckey >> 32) == kh) ? (uint32_t)ckey : 0u);
        if (lane == 0) {
          s_wsum[2 * warp] = ((unsigned long long)(uint32_t)wc << 32) | (uint32_t)wh;
          s_wsum[2 * warp + 1] = ((unsigned long long)kh << 32) | kl;
        }
      }
      __syncthreads();
      if (warp == 0) {
        const unsigned long long none = ((unsigned long long)kNoStep << 32) | (uint32_t)kNoStep;
        const unsigned long long a = lane < nwarps ? s_wsum[2 * lane] : none;
        const unsigned long long k = lane < nwarps ? s_wsum[2 * lane + 1] : 0ull;
        const int wc = (int)(a >> 32), wh = (int)(uint32_t)a;
        const int C = __reduce_min_sync(FULL, wc);
        const int H = __reduce_min_sync(FULL, wh);
        const uint32_t kh = __reduce_max_sync(FULL, wc == C ? (uint32_t)(k >> 32) : 0u);
        const uint32_t kl = layer ? __reduce_add_sync(FULL, wc == C ? (uint32_t)k : 0u)
                                  : __reduce_max_sync(FULL, (wc == C && (uint32_t)(k >> 32) == kh) ? (uint32_t)k : 0u);
        const unsigned long long A = ((unsigned long long)(uint32_t)C << 32) | (uint32_t)H;
        const unsigned long long K = ((unsigned long long)kh << 32) | kl;
        unsigned long long* slot = s_slots + (size_t)(fp * kMaxCluster + rank) * 2;
        if (cs == 1) {
          if (lane == 0) { slot[0] = A; slot[1] = K; }
        } else if (lane < cs) {
          st_cluster_u64(slot, (uint32_t)lane, A);
          st_cluster_u64(slot + 1, (uint32_t)lane, K);
        }
        if (lane == 0) s_flag[fp ^ 1] = INT_MAX;
      }
      if (cs > 1) { cluster_arrive(); cluster_wait(); } else { __syncthreads(); }   // the one cross-SM exchange
      if (trace && tid == 0) { tg3 = globaltimer(); tc3 = clock64(); }

      // ---------------------------------------------------------- global decision
      int P, H;
      unsigned long long K;
      {
        const unsigned long long none = ((unsigned long long)kNoStep << 32) | (uint32_t)kNoStep;
        const unsigned long long A = lane < cs ? s_slots[(size_t)(fp * kMaxCluster + lane) * 2] : none;
        const unsigned long long Kr = lane < cs ? s_slots[(size_t)(fp * kMaxCluster + lane) * 2 + 1] : 0ull;
        const int c = (int)(A >> 32), h = (int)(uint32_t)A;
        P = __reduce_min_sync(FULL, c);
        H = __reduce_min_sync(FULL, h);
        const uint32_t kh = __reduce_max_sync(FULL, c == P ? (uint32_t)(Kr >> 32) : 0u);
        const uint32_t kl = layer ? __reduce_add_sync(FULL, c == P ? (uint32_t)Kr : 0u)
                                  : __reduce_max_sync(FULL, (c == P && (uint32_t)(Kr >> 32) == kh) ? (uint32_t)Kr : 0u);
        K = ((unsigned long long)kh << 32) | kl;
      }
      if (sharded) {
        // the cluster's summary {P, H, K} goes to slot [cur & 1][shard] of every rank's mailbox as four LL words
        // (NVLink peer stores, no fence); warp 0 of every CTA polls its own mailbox for the world's summaries and
        // applies the same reduction as the cluster exchange
        const int mp = (int)(cur & 1u);
        const unsigned long long tag = (unsigned long long)cur << 32;
        if (rank == 0 && warp == 0 && lane < world) {
          unsigned long long* sl = d.peers[lane]->slot[mp][d.shard];
          st_relaxed_sys_u64(sl, tag | (uint32_t)P);
          st_relaxed_sys_u64(sl + 1, tag | (uint32_t)H);
          st_relaxed_sys_u64(sl + 2, tag | (uint32_t)(K >> 32));
          st_relaxed_sys_u64(sl + 3, tag | (uint32_t)K);
        }
        if (warp == 0) {
          int c = kNoStep, h = kNoStep;
          unsigned long long Kr = 0ull;
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
            c = (int)(uint32_t)w0; h = (int)(uint32_t)w1;
            Kr = ((unsigned long long)(uint32_t)w2 << 32) | (uint32_t)w3;
          }
          const int Pg = __reduce_min_sync(FULL, c);
          const int Hg = __reduce_min_sync(FULL, h);
          const uint32_t kh = __reduce_max_sync(FULL, c == Pg ? (uint32_t)(Kr >> 32) : 0u);
          const uint32_t kl = layer ? __reduce_add_sync(FULL, c == Pg ? (uint32_t)Kr : 0u)
                                    : __reduce_max_sync(FULL, (c == Pg && (uint32_t)(Kr >> 32) == kh) ? (uint32_t)Kr : 0u);
          // (own words: the next write comes after the next cluster barrier, which every thread reaches after
          // reading these)
          unsigned long long* s_world = reinterpret_cast<unsigned long long*>(s_misc + 32);
          if (lane == 0) {
            s_world[0] = ((unsigned long long)(uint32_t)Pg << 32) | (uint32_t)Hg;
            s_world[1] = ((unsigned long long)kh << 32) | kl;
          }
        }
        __syncthreads();
        const unsigned long long* s_world = reinterpret_cast<const unsigned long long*>(s_misc + 32);
        P = (int)(s_world[0] >> 32);
        H = (int)(uint32_t)s_world[0];
        K = s_world[1];
      }
      const bool event = P < kend && P < H;          // a post spike at t* = P
#ifdef SNN_LEAN_DEBUG
      if (tid == 0 && k0 >= 116) printf("EP r %d b %d k0 %d ka %d kend %d P %d H %d\n", rank, b, k0, ka, kend, P, H);
#endif
      const int k_last = event ? P : (H < kend ? H - 1 : kend - 1);   // last committed step

      // ---------------------------------------------------------- per-thread resolution
      auto undo_after = [&](int rel_keep) {           // undo logged LTD of steps k0 + rel > k0 + rel_keep
        while (nlog > 0) {
          const uint32_t e = s_log[(nlog - 1) * nthr + tid];
          if ((int)(e >> 16) <= rel_keep) break;
          if (e & 0x2000u) atomicAdd(s_w + (int)(e & 0x1FFFu) * wpr + wj, 1u << (fsh + (int)((e >> 14) & 3u) * Z::LW));
          --ltd_events;
          --nlog;
          ++eng_undo;
        }
      };
      uint32_t spk = 0u;                               // LAYER: own columns spiking at t*
      if (event) {
        const uint32_t W = 0xFFFFFFFFu - (uint32_t)K;
        // HARD: one spiker W; LAYER: every column that crossed at t* (K = their number, R7)
        const uint32_t nsp = layer ? (uint32_t)K : 1u;
        if (layer && cstep == P) spk = cmk;
        undo_after(P - k0);
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
          if (!(valid >> c & 1u)) continue;
          const bool me = layer ? ((spk >> c & 1u) != 0u) : (uint32_t)(cbase + col0 + jcol[c]) == W;
          // no crossing in [k0, t*) anywhere: the countdown only ran down (R6, R7), v is reset anyway
          const int cnt_p = max(cnt0[c] - (P - k0 + 1), 0);
          if (me) {
            // a lone spiker keeps t_ref; with >= 2 spikers every neuron, the spikers included, is inhibited (R7)
            v[c] = vreset; cnt[c] = nsp >= 2 ? max(t_ref, t_inh) : t_ref;
            if (rec_out) atomicOr(&d.raster_out[(size_t)P * d.nwe + ((col0 + jcol[c]) >> 5)], 1u << ((col0 + jcol[c]) & 31));
          } else {
            v[c] = vreset; cnt[c] = max(cnt_p, t_inh);
          }
        }
        img_spikes += (int)nsp;
      } else if (p_done > k_last) {                    // undo log full somewhere: replay [k0 + 1, k_last]
        ++eng_resim;
        undo_after(0);
#pragma unroll
        for (int c = 0; c < CPT; ++c) { v[c] = v1[c]; cnt[c] = cnt1[c]; }
        const int t_unused = 0; (void)t_unused;
        for (int k2 = k0 + 1; k2 <= k_last; ++k2) {
          const int x2 = k2 - ka;
          int S[CPT];
#pragma unroll
          for (int c = 0; c < CPT; ++c) S[c] = 0;
          for (int r = (int)s_offs[x2]; r < (int)s_offs[x2 + 1]; ++r) {
            const int i = (int)(s_rraw[r] & 0xFFFFu);
            const uint32_t w = s_w[i * wpr + wj];
#pragma unroll
            for (int c = 0; c < CPT; ++c) S[c] += (int)((w >> (fsh + c * Z::LW)) & FMASK);
          }
#pragma unroll
          for (int c = 0; c < CPT; ++c) if (c == dslot) S[c] = s_dS[k2 - tk0];   // k2 <= k_last <= kcov
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            if (!(valid >> c & 1u)) continue;
            if (cnt[c] > 0) --cnt[c]; else lif.step_t<FIXED>(v[c], S[c]);
          }
          const int t = tbase + k2;
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            if (!(dmask >> c & 1u) || (t - lpost[c]) >= L_dep) continue;
            const uint32_t thr = s_dep[t - lpost[c]];
            const int jg = cbase + col0 + jcol[c];
            const int shc = fsh + c * Z::LW;
            for (int r = (int)s_offs[x2]; r < (int)s_offs[x2 + 1]; ++r) {
              const int i = (int)(s_rraw[r] & 0xFFFFu);
              const uint4 u = philox((uint32_t)t, (uint32_t)i, (uint32_t)(jg >> 2), TAG_LTD, seed);
              if (pick(u, jg & 3) <= thr) {
                uint32_t* pw = s_w + i * wpr + wj;
                if ((*pw >> shc) & FMASK) atomicSub(pw, 1u << shc);
                ++ltd_events;
              }
            }
          }
        }
      }
      // LTD trials of the committed steps (draws with D < L_dep, R20)
#pragma unroll
      for (int c = 0; c < CPT; ++c) {
        if (!(dmask >> c & 1u)) continue;
        const int last = min(k_last, lpost[c] + L_dep - 1 - tbase);
        if (last >= k0) ltd_trials += s_offs[last + 1 - ka] - s_offs[k0 - ka];
      }
      nlog = 0;

      // ---------------------------------------------------------- LTP at t* in the winner's CTA (eq.(6))
      if (event && layer) {
        // LAYER: every CTA holding spikers brings its input timers up to t*, writes back its deferred table through
        // t*, takes the lowest spiking column as its new deferred column and runs the eq.(6) LTP of all of its
        // spikers (each thread owns its input rows for every spiker: no word is written by two threads)
        const int tP = tbase + P;
        if (tid == 0) s_misc[37] = 0;
        __syncthreads();
#pragma unroll
        for (int c = 0; c < CPT; ++c)
          if (spk >> c & 1u) { lpost[c] = tP; s_spk[atomicAdd(&s_misc[37], 1)] = jcol[c]; }   // after LTD at t*
        __syncthreads();
        const int nsl = s_misc[37];
        if (nsl > 0) {                                                        // CTA-uniform
          if (tvalid) dtab_apply(P);
          lpre_catch_up(P - ka);
          __syncthreads();
          dtab_clear();
          int wmin = INT_MAX;
          for (int q = 0; q < nsl; ++q) wmin = min(wmin, s_spk[q]);
          Wd = wmin; d_lp = tP;
          const bool tab = P + 1 < kend && dtab_draw(P + 1);
          for (int grp = tid; grp < nq4; grp += nthr) {
            for (int q = 0; q < nsl; ++q) {
              const int Ws = s_spk[q];
              const int Wg = cbase + col0 + Ws;
              const int ww = Ws / CPW, wsh = (Ws % CPW) * BITS;
              const uint4 u = philox((uint32_t)tP, (uint32_t)Wg, (uint32_t)grp, TAG_LTP, seed);   // eq.(6), R13
#pragma unroll
              for (int r = 0; r < 4; ++r) {
                const int i = 4 * grp + r;
                if (i >= n_in) break;
                const int lpi = s_lpre[i];
                if (lpi < 0) continue;
                const int D = tP - lpi;                                        // R10: Dt = D >= 0
                if (D >= L_pot) continue;
                ++ltp_trials;
                if (pick(u, r) <= s_pot[D]) {
                  ++ltp_events;
                  uint32_t* pw = s_w + i * wpr + ww;            // rows 4 grp .. 4 grp + 3 are this thread's alone
                  const uint32_t wv = *pw;
                  if (((wv >> wsh) & FMASK) < (uint32_t)qmax) *pw = wv + (1u << wsh);
                }
              }
            }
          }
          __syncthreads();
          if (tab) { dtab_sums(); __syncthreads(); }
        }
      }
      if (event && !layer) {
        const int Wl = (int)(0xFFFFFFFFu - (uint32_t)K) - cbase - col0;     // winner's local column
        const int tP = tbase + P;
#pragma unroll
        for (int c = 0; c < CPT; ++c)
          if ((valid >> c & 1u) && jcol[c] == Wl) lpost[c] = tP;             // after LTD at t* (R14)
        if (Wl >= 0 && Wl < ncols) {                                           // CTA-uniform
          // phase 1: the previous deferred column's eq.(7) events through t* (old last_post, R14) and the input
          // spike timers through t* (no barrier before: the catch-up reads only the staged window and writes only
          // s_lpre; the table write-back touches only the deferred column's fields, atomically)
          if (tvalid) dtab_apply(P);
          lpre_catch_up(P - ka);                                               // last_pre includes step t*
          __syncthreads();
          if (trace && tid == 0) tph[0] = clock64();
          // phase 2: LTP of the winner (eq.(6)) next to the eq.(7) draws of its table (it is the new deferred
          // column, last_post = t*) and the clearing of the retired table's masks
          dtab_clear();
          Wd = Wl; d_lp = tP;
          const bool tab = P + 1 < kend && dtab_draw(P + 1);
          if (trace && tid == 0) tph[1] = clock64();
          const int Wg = cbase + col0 + Wl;
          const int ww = Wl / CPW, wsh = (Wl % CPW) * BITS;
          for (int grp = tid; grp < nq4; grp += nthr) {
            const uint4 u = philox((uint32_t)tP, (uint32_t)Wg, (uint32_t)grp, TAG_LTP, seed);
#pragma unroll
            for (int r = 0; r < 4; ++r) {
              const int i = 4 * grp + r;
              if (i >= n_in) break;
              const int lpi = s_lpre[i];
              if (lpi < 0) continue;
              const int D = tP - lpi;                                          // R10: Dt = D >= 0
              if (D >= L_pot) continue;
              ++ltp_trials;
              if (pick(u, r) <= s_pot[D]) {
                ++ltp_events;
                uint32_t* pw = s_w + i * wpr + ww;              // row i is this thread's alone during LTP
                const uint32_t wv = *pw;
                if (((wv >> wsh) & FMASK) < (uint32_t)qmax) *pw = wv + (1u << wsh);
              }
            }
          }
          if (trace && tid == 0) tph[2] = clock64();
          __syncthreads();
          if (trace && tid == 0) tph[3] = clock64();
          if (tab) { dtab_sums(); __syncthreads(); }   // phase 3: the table's sums read the codes after LTP
          if (trace && tid == 0) tph[4] = clock64();
        }
      }
      if (trace && tid == 0 && ep < d.trace_cap) {
        unsigned long long* rec = trace + (size_t)ep * 8;
        rec[0] = ((unsigned long long)b << 32) | (unsigned)k0 | ((unsigned long long)min(s_trsteps[fp * 3], 0xFFFF) << 48);
        rec[1] = ((unsigned long long)(event ? 1 : 2) << 32) | (unsigned)P |
                 ((unsigned long long)min(s_trsteps[fp * 3 + 1], 0xFFFF) << 48);
        rec[2] = tg0; rec[3] = s_trmax[fp]; rec[5] = tg3;
        rec[4] = (event ? (unsigned long long)(0xFFFFFFFFu - (uint32_t)K) : 0xFFFFFFFFull) |   // winner column
                 ((unsigned long long)min(s_trsteps[fp * 3 + 2], 0xFFFF) << 48);
        rec[6] = s_trloop[fp];   // slowest warp: loop | draws | LTD events | integration+LIF (cycles / 16, 16 bits each)
        if (!kTraceCycles) {     // winner's CTA: the three phases after the exchange (cycles / 8 after it, 16 bits each)
          rec[6] = 0ull;
          if (tph[0] > tc3)
            for (int q = 0; q < 4; ++q) rec[6] |= min((tph[q + 1] - tph[q]) >> 3, 0xFFFFull) << (48 - 16 * q);
        }
        s_trcross[fp] = ~0ull;
        tph[0] = tph[1] = tph[2] = tph[3] = tph[4] = 0ull;
        rec[7] = globaltimer();
        s_trmax[fp] = 0ull; s_trloop[fp] = 0ull; s_trdepth[fp] = 0;
        s_trsteps[fp * 3] = s_trsteps[fp * 3 + 1] = s_trsteps[fp * 3 + 2] = 0;   // reused at epoch ep + 2 (after two barriers)
      }
      k0 = k_last + 1;
      ++ep;
      ++eng_epochs;
    }  // epochs
    if (tvalid) dtab_retire(min(T - 1, kcov));      // every table step is committed by now

    if (rank == 0 && tid == 0) {
      post_sum += (unsigned long long)img_spikes;
      if (d.spike_counts) d.spike_counts[b] = img_spikes;
    }
    if (last_img) {
#pragma unroll
      for (int c = 0; c < CPT; ++c)
        if (valid >> c & 1u) {
          const int jg = col0 + jcol[c];
          d.v[jg] = v[c]; d.cnt[jg] = cnt[c]; d.last_post[jg] = lpost[c];
        }
      __syncthreads();
      if (kb > ka) lpre_catch_up(kb - 1 - ka);
      __syncthreads();
      if (rank == 0) for (int i = tid; i < n_in; i += nthr) d.last_pre[i] = s_lpre[i];
    } else if (kb > ka) {
      // the next image resets the timers (R5); nothing to finish
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
#ifdef SNN_LEAN_DEBUG
  if (tid == 0) printf("END r %d\n", rank);
#endif
  if (sharded && rank == 0 && tid == 0) d.mbox->seq = seq0 + (uint32_t)ep;   // every CTA read seq0 long ago
  if (cs > 1) { cluster_arrive(); cluster_wait(); }
}

// ====================================================================== host launchers
template <int BITS, int CPT, bool FIXED, bool SH, bool LAY>
static cudaError_t lean_launch_t(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, cudaStream_t s,
                                 int* occupancy_out) {
  auto* kern = present_lean_kernel<BITS, CPT, FIXED, SH, LAY>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (cs > 8) {
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
  }
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
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
  if (occupancy_out) {
    if (cs == 1) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occupancy_out, kern, nthr, smem);
    return cudaOccupancyMaxActiveClusters(occupancy_out, kern, &cfg);
  }
  return cudaLaunchKernelEx(&cfg, kern, lp);
}

// sh: 0 unsharded HARD, 1 sharded HARD, 2 unsharded LAYER
template <int BITS, int CPT>
static cudaError_t lean_dispatch_f(int fixed, int sh, const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem,
                                   cudaStream_t s, int* occ) {
  if (sh == 2)
    return fixed ? lean_launch_t<BITS, CPT, true, false, true>(lp, n_nets, cs, nthr, smem, s, occ)
                 : lean_launch_t<BITS, CPT, false, false, true>(lp, n_nets, cs, nthr, smem, s, occ);
  if (sh == 1)
    return fixed ? lean_launch_t<BITS, CPT, true, true, false>(lp, n_nets, cs, nthr, smem, s, occ)
                 : lean_launch_t<BITS, CPT, false, true, false>(lp, n_nets, cs, nthr, smem, s, occ);
  return fixed ? lean_launch_t<BITS, CPT, true, false, false>(lp, n_nets, cs, nthr, smem, s, occ)
               : lean_launch_t<BITS, CPT, false, false, false>(lp, n_nets, cs, nthr, smem, s, occ);
}

static cudaError_t lean_dispatch(int bits, int cpt, int fixed, int sh, const LaunchParams& lp, int n_nets, int cs,
                                 int nthr, size_t smem, cudaStream_t s, int* occ) {
  if (bits == 2) {
    if (cpt == 4) return lean_dispatch_f<2, 4>(fixed, sh, lp, n_nets, cs, nthr, smem, s, occ);
    if (cpt == 1) return lean_dispatch_f<2, 1>(fixed, sh, lp, n_nets, cs, nthr, smem, s, occ);
    return lean_dispatch_f<2, 2>(fixed, sh, lp, n_nets, cs, nthr, smem, s, occ);
  }
  if (bits == 4) {
    if (cpt == 1) return lean_dispatch_f<4, 1>(fixed, sh, lp, n_nets, cs, nthr, smem, s, occ);
    return lean_dispatch_f<4, 2>(fixed, sh, lp, n_nets, cs, nthr, smem, s, occ);
  }
  return lean_dispatch_f<8, 1>(fixed, sh, lp, n_nets, cs, nthr, smem, s, occ);
}

cudaError_t query_max_clusters_lean(int bits, int cpt, int fixed, int cs, int nthr, size_t smem, int* out) {
  LaunchParams lp{};
  return lean_dispatch(bits, cpt, fixed, 0, lp, 1, cs, nthr, smem, 0, out);
}

cudaError_t launch_present_lean(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, int bits, int cpt,
                                int fixed, int sharded, int layer, cudaStream_t s) {
  if (sharded && layer) return cudaErrorNotSupported;     // (the runtime never selects it)
  return lean_dispatch(bits, cpt, fixed, layer ? 2 : (sharded ? 1 : 0), lp, n_nets, cs, nthr, smem, s, nullptr);
}

}  // namespace snn
