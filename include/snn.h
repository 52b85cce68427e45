/*
 * snn.h -- C ABI of the B200 (sm_100a) simulate-and-learn path of
 *   She, Long & Mukhopadhyay, "Fast and Low-Precision Learning in GPU-Accelerated Spiking
 *   Neural Network", DATE 2019.  Paper text: /root/reference/PAPER.md, cited as P:<line>.
 *
 * One call of snn_present* runs, for every image and every timestep t, the four steps of the
 * paper's per-timestep loop (Fig. 2 flowchart, §III-A) entirely in CUDA kernels:
 *   (a1) Poisson rate encoding of the 8-bit image        P:88 §III-B
 *   (a2) synaptic integration I_a = sum_n g_{n,a} v_pre  P:83 eq.(3)
 *   (a3) LIF update dv/dt = a + b v + c I, reset          P:83 eqs.(1)(2), P:90 constants
 *   (a4) winner-take-all lateral inhibition for t_inh     P:88 §III-B
 *   (a5) stochastic STDP, eqs.(6)(7), dG = 1 LSB          P:85 §II-C, §III-C
 *   (a6) deterministic STDP arm, eqs.(4)(5) + rounding     P:84 §II-B, eq.(8)
 * The exact semantics (every reading of a silent or garbled passage, the Philox counter
 * layout, the fixed-point recipe) are DESIGN.md §2-§3.
 *
 * Conventions
 *  - Every function returns SNN_OK (0) or a negative SNN_E* code; snn_last_error() returns a
 *    thread-local message for the last failure on the calling thread.
 *  - The caller owns every buffer it passes; the library never retains a caller pointer past
 *    the call (asynchronous calls: past the completion of the work they enqueue, see SNN_ASYNC).
 *  - "host or device" pointers are classified with cudaPointerGetAttributes; host memory may be
 *    pageable or pinned.
 *  - A handle owns all of its device memory and is bound to the device current at snn_create.
 *    Handles are not thread-safe; distinct handles may be used from distinct threads.
 *  - Weights persist across presentations (online learning).  v, refractory counters and
 *    spike timers are reset at the start of each presentation unless SNN_KEEP_STATE (R5).
 *
 * Differences from the call list of SURVEY.md §8(b) (which this header otherwise follows):
 *  - snn_present_many takes an n_images argument: each handle presents a batch of images in the one
 *    launch (the ensemble C5 runs 8 networks x B images per call), not one image per handle.
 *  - snn_create_sharded(..., nccl_unique_id) became snn_create_shard + snn_shard_ipc_handle /
 *    snn_shard_connect (multi-process) or snn_shard_link (one process): the exchange step is a
 *    16-byte per-epoch summary (event engines) or a per-step WTA summary (per-step engine) written by the
 *    kernel itself into every rank's device mailbox (NVLink peer stores), so there is no
 *    NCCL communicator to bootstrap.  The only
 *    host-side collective is the caller's all_gather of the 64-byte IPC handles.  SNN_ENCCL is kept
 *    (reserved) so that the error-code values of §8(b) do not shift.
 *  - Added beyond §8(b): snn_present_batch / snn_present_ex (batches, raster input, KEEP_STATE),
 *    state/trace/info accessors, bits = 16 (R27) and bits = 32 (binary32 conductance, R28), and the
 *    NEXT-1 / NEXT-4 entry points below.
 */
#ifndef SNN_H
#define SNN_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SNN_OK       0
#define SNN_EINVAL  (-1)   /* invalid argument or parameter                       */
#define SNN_ENOMEM  (-2)   /* host or device allocation failed                    */
#define SNN_ECUDA   (-3)   /* CUDA runtime error (message in snn_last_error)      */
#define SNN_ENCCL   (-4)   /* reserved (never returned): the shard exchange uses no NCCL, see below */
#define SNN_ESIZE   (-5)   /* caller buffer too small, or network exceeds the on-chip capacity */
#define SNN_ECOOP   (-6)   /* cluster / co-residency launch not possible          */

/* wta_mode */
#define SNN_WTA_HARD   0   /* at most one spike per step: the largest v - v_th wins, ties -> lowest j (R7) */
#define SNN_WTA_LAYER  1   /* every crossing neuron spikes (one-to-one inhibitory layer, R7)              */
/* inh_mode */
#define SNN_INH_RESET  0   /* inhibited neurons are reset to v_reset and held for t_inh steps */
#define SNN_INH_HOLD   1   /* inhibited neurons keep v and are held for t_inh steps           */
/* stdp_mode */
#define SNN_STDP_STOCH 0   /* eqs.(6)(7) gate a one-LSB step ("dG is set to 1/2^n")     */
#define SNN_STDP_DET   1   /* eqs.(4)(5) at each post spike, rounded to the grid (R16)        */
/* rounding (deterministic arm, "three available rounding options") */
#define SNN_ROUND_TRUNC   0
#define SNN_ROUND_NEAREST 1
#define SNN_ROUND_STOCH   2   /* eq.(8) */
/* membrane_mode */
#define SNN_MEM_FP32   0   /* explicit fmaf recipe */
#define SNN_MEM_FIXED  1   /* Q15.16 integer recipe */

/* Parameter block.  Field order and types are part of the ABI. */
typedef struct snn_params {
  /* LIF, §III-D: a=-6.77, b=-0.0989, c=0.314, V_th=-60.2, V_reset=-74.7, v_init=-70.0 */
  double a, b, c, v_th, v_reset, v_init;
  double dt_ms;          /* Euler step, ms (R1: 1.0)                                   */
  double v_spike;        /* pre-synaptic "voltage spike" v_pre of eq.(3) (R3: 2.0)      */
  double i_ext;          /* constant external current, test hook (0)                   */
  int32_t t_ref_steps;   /* refractory steps after a spike (R6: 5)                     */
  int32_t t_inh_steps;   /* lateral-inhibition steps, "t_inh" (R7: 10)            */
  int32_t wta_mode, inh_mode;
  double f_min_hz, f_max_hz;   /* encoder range, P:88 / Table I                         */
  int32_t stdp_mode, rounding;
  int32_t t_ltp_steps;   /* deterministic arm LTP window (R16: 20)                     */
  int32_t membrane_mode;
  double gamma_pot, tau_pot, gamma_dep, tau_dep;        /* eqs.(6)(7), Table I (ms)      */
  double alpha_p, beta_p, alpha_d, beta_d, g_min, g_max; /* eqs.(4)(5), Table I "16 bit" */
  int32_t frac_bits;     /* 0 = bits (LSB = 2^-bits); Q1.7-style grids: 7       */
  int32_t init_mode;     /* 0: uniform codes from Philox TAG_INIT (R4)                 */
  uint64_t init_seed;
  int32_t cluster_size;  /* 0 = auto; else CTAs per network (1..16)                    */
  int32_t engine;        /* SNN_ENGINE_EVENT (0, default) or SNN_ENGINE_STEP (1) */
} snn_params;

/* engine: both give bit-identical results */
#define SNN_ENGINE_EVENT 0   /* one cluster exchange per post-spike epoch; T <= 32767 */
#define SNN_ENGINE_STEP  1   /* one cluster exchange per timestep */
#define SNN_ENGINE_EVENT_GENERAL 2   /* the event engine's general kernel even where the lean one applies */
/* SNN_ENGINE_EVENT runs the lean kernel for HARD WTA + RESET inhibition + stochastic STDP
 * on an unsharded network (the paper's default mode) and the general event kernel otherwise. */

/* Table I rows */
#define SNN_PRESET_2B  0
#define SNN_PRESET_4B  1
#define SNN_PRESET_8B  2
#define SNN_PRESET_16B 3   /* Table I "16 bit" row: use with bits = 16 (R27) */
#define SNN_PRESET_HF  4   /* "high frequency": 5-78 Hz, tau_pot 80, tau_dep 5 */
int snn_params_preset(snn_params* p, int preset);

typedef struct snn_handle snn_handle;

/* Create a network n_in -> n_exc with `bits`-bit conductance codes (2, 4, 8 or 16), or with IEEE binary32
 * conductances (bits = 32).
 * 16 bits (NEXT-2, "For 16-bit ... after floating point calculation of change in conductance dG,
 * the result is rounded"; R27): every STDP event (stochastic arm) moves the code by the
 * eq.(4)/(5) magnitude rounded by `rounding` instead of one LSB; 16-bit handles run on the per-step
 * engine (SNN_ENGINE_STEP is selected automatically); they shard on it (snn_create_shard) and infer on it
 * (snn_infer, unsharded handles).
 * 32 bits (NEXT-2, "32-bit floating-point"; R28): every conductance is a binary32 G in
 * [g_min, g_max]; integration sums G in binary32 (I = v_spike * sum G); an STDP event (stochastic arm: gated
 * by the eqs.(6)(7) draw; deterministic arm: R16 window) sets G = binary32(G +- dG) with dG = eq.(4)/(5) in
 * binary64 by R28's exp recipe, clamped.  Requires membrane_mode = SNN_MEM_FP32 and rounding =
 * SNN_ROUND_NEAREST (else SNN_EINVAL); per-step engine; one cluster holds 784 -> <= 512 columns (227 KB per
 * CTA), larger networks run column-sharded (snn_create_shard).
 * Conductances are initialised on the device (R4).  SNN_ESIZE if the network does not fit the
 * on-chip layout.  *out receives the handle. */
int snn_create(int n_in, int n_exc, int bits, const snn_params* p, snn_handle** out);
int snn_destroy(snn_handle* h);

/* Stream used by every subsequent call on h (a cudaStream_t; NULL = the handle's own stream). */
int snn_set_stream(snn_handle* h, void* cuda_stream);
/* Block until all work enqueued on h has finished. */
int snn_synchronize(snn_handle* h);

/* flags */
#define SNN_RASTER_INPUT  1   /* `input` is a T x ceil(n_in/32) u32 input spike raster (encoder bypassed) */
#define SNN_KEEP_STATE    2   /* keep v / counters / timers; steps are numbered t0 .. t0+T-1              */
#define SNN_RECORD_INPUT  4   /* also record the input raster of the last image (snn_get_input_raster)    */
#define SNN_ASYNC         8   /* return after enqueueing; host buffers must stay valid until synchronize  */
#define SNN_FLOOR_PROBE  16   /* benchmark probe (results are discarded, weights untouched): the same launch
                                 shape doing only the synchronisation skeleton -- per step (per-step engine)
                                 or per epoch, with the handle's mean epochs per image so far (lean kernel) */

/* Present one image (n_in bytes, host or device) for T steps with learning on ("Each image is
 * presented to the network for t_learn ms").  `seed` keys every random draw of the presentation. */
int snn_present(snn_handle* h, const uint8_t* image, int T, uint64_t seed);

/* Present n_images images back to back in ONE kernel launch (weights stay resident on chip
 * between images).  images: n_images x n_in bytes; seeds: n_images (both host or device).
 * spike_counts (optional, host or device, n_images int32): post spikes per image. */
int snn_present_batch(snn_handle* h, const uint8_t* images, int n_images, int T, const uint64_t* seeds,
                      int32_t* spike_counts, int flags);

/* General form: input is an image (n_in bytes) or, with SNN_RASTER_INPUT, a T x ceil(n_in/32)
 * u32 raster (host or device); t0 is the first step index (only meaningful with SNN_KEEP_STATE). */
int snn_present_ex(snn_handle* h, const void* input, int T, uint64_t seed, int flags, int t0);

/* Test hook: present a given input raster (T x ceil(n_in/32) u32), encoder bypassed. */
int snn_present_raster(snn_handle* h, const uint32_t* raster, int T, uint64_t seed);

/* Ensemble: n independent handles (equal n_in, n_exc, cluster size; bits and parameters may
 * differ) each present n_images images in ONE launch (linked shards of one world: all of them,
 * see snn_shard_link).  images[k]: n_images x n_in bytes and
 * seeds[k]: n_images seeds for handle k (arrays of host pointers to host or device buffers). */
int snn_present_many(snn_handle* const* hs, int n, const uint8_t* const* images, int n_images, int T,
                     const uint64_t* const* seeds);

/* Readout.  codes: n_in x n_exc codes, row-major [i][j], one code per byte (bits <= 8) or one
 * little-endian uint16 per code (bits = 16); G = code * 2^-frac_bits.  bits = 32: one little-endian binary32
 * G per synapse (set: every G finite and in [g_min, g_max], else SNN_EINVAL).  cap / n are in BYTES. */
int snn_get_weights(snn_handle* h, uint8_t* codes, size_t cap);
int snn_set_weights(snn_handle* h, const uint8_t* codes, size_t n);
/* Output raster of the last presented image: T x ceil(n_exc/32) u32, bit j%32 of word j/32. */
int snn_get_spikes(snn_handle* h, uint32_t* raster, size_t cap_words);
/* Input raster of the last presented image (requires SNN_RECORD_INPUT): T x ceil(n_in/32) u32. */
int snn_get_input_raster(snn_handle* h, uint32_t* raster, size_t cap_words);
/* State blob: int32 {n_in, n_exc, t_next, membrane_mode}, v[n_exc] (fp32 bits
 * or Q15.16), cnt[n_exc], last_post[n_exc], last_pre[n_in]. */
size_t snn_state_bytes(const snn_handle* h);
int snn_get_state(snn_handle* h, void* buf, size_t cap);
int snn_set_state(snn_handle* h, const void* buf, size_t n);
/* Counters accumulated since the last snn_reset_stats: [0] sum_t act(t) (active input rows),
 * [1] post spikes, [2] LTD trials, [3] LTD events, [4] LTP trials, [5] LTP events,
 * [6] images presented, [7] steps simulated; event engine only: [8] epochs
 * (cluster exchanges), [9] speculation stops on a full undo log, [10] re-simulations,
 * [11] speculated column-steps, [12] undone LTD events; [13..15] reserved (0). */
/* Kernel timing (bench.py roofline): with profiling on, every presentation records CUDA events on the
 * handle's stream immediately before and after its presentation kernel (the pre-pass kernels of the
 * event engine are outside the pair).  snn_get_profile synchronises the stream and returns the summed
 * kernel milliseconds and the number of kernels since the last call (or snn_set_profile), then resets. */
int snn_set_profile(snn_handle* h, int on);
int snn_get_profile(snn_handle* h, double* kernel_ms, int64_t* kernels);
#define SNN_NSTATS 16
int snn_get_stats(snn_handle* h, uint64_t stats[SNN_NSTATS]);
int snn_reset_stats(snn_handle* h);
/* Introspection: [0] cluster size, [1] threads per CTA, [2] dynamic smem bytes per CTA,
 * [3] words per weight row in a CTA slice, [4] q_max, [5] L_pot, [6] L_dep, [7] kernel launches so far,
 * [8] engine, [9] columns per thread (event engine), [10] on-chip row window, [11] LTD undo-log depth,
 * [12] first global column (col_base), [13] columns of the whole network, [14] world, [15] shard,
 * [16] 1 if the lean event kernel runs, [17] its dynamic smem bytes per CTA. */
#define SNN_NINFO 18
int snn_get_info(const snn_handle* h, int64_t info[SNN_NINFO]);

/* Tracing: with max_epochs > 0 the event engine records, per CTA and epoch,
 * 8 u64 values: {image<<32 | k0, kind<<32 | P, t_spec_start, t_spec_end (max over warps),
 * t_summary, t_exchanged, t_committed, t_end} (%globaltimer ns; kind 1 = post spike, 2 = no
 * event / log stop, 0 = end of window).  snn_get_trace copies cluster_size x max_epochs x 8
 * values of the last presentation call.  0 disables tracing. */
int snn_set_trace(snn_handle* h, int max_epochs);
int snn_get_trace(snn_handle* h, uint64_t* out, size_t cap);

/* ---- Column sharding of ONE network across ranks.
 * The n_exc_total post-synaptic columns are split into `world` contiguous slices on 32-column
 * boundaries: shard r owns columns [32*floor(r*G/world), 32*floor((r+1)*G/world)) with
 * G = ceil(n_exc_total/32) (G >= world required).  A shard handle is a network of its own columns
 * whose random draws (R13: init, LTD, LTP, rounding) and WTA keys (R7) use GLOBAL column indices, so
 * the union of the shards reproduces the unsharded network bit for bit.  The encoder and the input
 * spike timers are replicated (every shard draws the same inputs from the same seeds).  Per epoch of
 * the event engine each shard publishes a 16-byte summary (earliest crossing step,
 * crossing count, best WTA key) into every shard's mailbox in device memory (peer stores over NVLink)
 * and every shard applies the same reduction: the exchange step of P:88 §III-B's lateral inhibition
 * across GPUs.  On the per-step engine (SNN_ENGINE_STEP; 16-bit codes and binary32 conductances always run
 * there) the exchange is per step: each shard publishes its cluster's best WTA key (HARD) or spiker count
 * (LAYER) the same way, so a 784 -> 6400 network at 16 / 32 bits (10 / 20 MB, beyond one cluster's shared
 * memory) runs as 4 / 7 shards.  All shards of a world must run the same presentation calls
 * (inputs, seeds, T, flags) in the same order; a rank that stops answering makes the others trap
 * after 20 s instead of hanging.
 * Readouts (weights, spikes, state) of a shard cover its own columns: n_in x n_exc_local codes, a
 * T x ceil(n_exc_local/32) raster, state with n_exc = n_exc_local.  Stats [2..5] count the shard's own
 * trials/events; [0], [1], [6], [7] are the network's (identical on every shard). */
#define SNN_IPC_HANDLE_BYTES 64
int snn_create_shard(int n_in, int n_exc_total, int bits, const snn_params* p, int shard, int world,
                     snn_handle** out);
/* Multi-process (one rank per GPU): export this shard's mailbox as a CUDA IPC handle
 * (SNN_IPC_HANDLE_BYTES bytes into out), gather all ranks' handles (e.g. torch.distributed
 * all_gather), then connect with the world's handles in rank order (world x SNN_IPC_HANDLE_BYTES). */
int snn_shard_ipc_handle(snn_handle* h, void* out, size_t cap);
int snn_shard_connect(snn_handle* h, const void* handles, size_t n_bytes);
/* Single process: link shards 0..world-1 directly (hs[r] is shard r).  Shards on one device must be
 * presented together with snn_present_many (one launch keeps every shard co-resident); shards on
 * distinct peer-capable devices may be presented from one thread each. */
int snn_shard_link(snn_handle* const* hs, int world);

/* ---- NEXT-1: labelling and inference with frozen weights (R21-R23).
 * P:88 §III-B: "After learning is complete, the first 1000 images in the test set are used to label
 * all the neurons in the first layer. The rest of the test set, which contains 9000 images, are used
 * for inference."
 *
 * snn_infer: present each of n_images images (n_images x n_in bytes) for T steps with the handle's
 * current weights FROZEN (steps 1-4 of the loop, no STDP, R21): encoder, integration, LIF and WTA as
 * in snn_present, state reset per image (R5), image k keyed by seeds[k].  counts (n_images x n_exc u32,
 * row-major [k][j]) receives the number of spikes of neuron j during image k.  The images are
 * independent and run in parallel (one CTA per image at a time, weights streamed from L2).
 * Weights, state, rasters and the learning stats are not touched; stats [0]/[1] of snn_get_stats are
 * not updated either (inference counters: snn_get_infer_stats).  All pointers host or device (the call
 * stages host buffers); SNN_ASYNC returns after enqueueing.  T <= 65535; n_exc <= 7168;
 * unsharded handles only.  Errors: SNN_EINVAL (arguments), SNN_ESIZE (n_exc too large), SNN_ECUDA.
 * 16-bit codes and binary32 conductances (bits 16 / 32) run their inference on the per-step engine
 * instead: the same semantics, the images one after another on the handle's cluster (synchronous).
 * snn_get_infer_stats: [0] sum over images and steps of active input rows, [1] post spikes, [2] column-
 * steps that ran the eqs.(1)(2) update (neither refractory nor inhibited: the LIF work that cannot be
 * skipped; counted by the <= 8-bit path only), since the handle was created.
 *
 * snn_label (R22): labels[j] (n_exc int32) = the class c maximising the MEAN count of neuron j over
 * the labelling images of class c (counts: n_images x n_exc u32, classes: n_images int32 in
 * [0, n_classes)); ties -> lowest class; -1 for a neuron that never spiked.  n_classes <= 64.
 * snn_classify (R23): pred[k] (n_images int32) = the class whose labelled neurons have the highest
 * MEAN count in image k; ties -> lowest class; -1 if no labelled neuron spiked.  Ratios are compared
 * exactly (integer cross products).  Pointers host or device; synchronous. */
int snn_infer(snn_handle* h, const uint8_t* images, int n_images, int T, const uint64_t* seeds, uint32_t* counts,
              int flags);
int snn_get_infer_stats(snn_handle* h, uint64_t stats[3]);
/* snn_infer_many: snn_infer for n per-step-engine handles in ONE launch (bits 16 / 32, or SNN_ENGINE_STEP):
 * independent networks and, what snn_infer cannot do, the linked shards of one column-sharded network (every
 * shard of its world must be in the call; each shard counts its own columns).  images[k] / seeds[k] /
 * counts[k] (n_images x n_exc_k u32) per handle, host or device.  Synchronous; weights and state untouched.
 * SNN_EINVAL for event-engine handles or an incomplete world. */
int snn_infer_many(snn_handle* const* hs, int n, const uint8_t* const* images, int n_images, int T,
                   const uint64_t* const* seeds, uint32_t* const* counts);
int snn_label(snn_handle* h, const uint32_t* counts, int n_images, const int32_t* classes, int n_classes,
              int32_t* labels);
int snn_classify(snn_handle* h, const uint32_t* counts, int n_images, const int32_t* labels, int n_classes,
                 int32_t* pred);

/* ---- NEXT-4: the Fig. 4 workload (R24-R26).
 * P:92 §IV-A: "We first evaluate the accuracy of the spiking neuron simulation (no learning) considering
 * an SNN of 10^3 LIF neurons and 10^4 synapses."
 * snn_sparse_run simulates n_trials independent trials of a sparse recurrent network of n_lif LIF
 * neurons with the handle's parameter block (LIF recipe, t_ref, encoder rates, bits -> LSB) and NOT its
 * weights: sources 0..n_in-1 are the rate-coded pixels of images[k] (the encoder of snn_present, seeds[k]),
 * sources n_in..n_in+n_lif-1 are the neurons (their spikes arrive one step later, R25).  Synapses CSR by
 * source: src_off[n_in + n_lif + 1] (int32, src_off[0] = 0, non-decreasing), tgt[n_syn] (u16 < n_lif),
 * q[n_syn] (u8 codes <= q_max).  Per step S_j = sum of codes of synapses from active sources; LIF with
 * refractory; no WTA, no inhibition, no STDP (R26).  counts: n_trials x n_lif u32 spikes per neuron;
 * raster (optional, may be NULL): n_trials x T x ceil(n_lif/32) u32.  Pointers host or device (graph
 * validated on the host: SNN_EINVAL).  n_lif <= 16384, T <= 2^30.  Synchronous unless SNN_ASYNC.
 * snn_get_sparse_stats: [0] input spikes, [1] neuron spikes, summed over all sparse runs of the handle. */
int snn_sparse_run(snn_handle* h, int n_lif, const int32_t* src_off, const uint16_t* tgt, const uint8_t* q,
                   const uint8_t* images, int n_trials, int T, const uint64_t* seeds, uint32_t* counts,
                   uint32_t* raster, int flags);
int snn_get_sparse_stats(snn_handle* h, uint64_t stats[2]);

const char* snn_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* SNN_H */
