// snn_internal.h -- descriptor shared by the host runtime (snn_api.cu) and the kernels
// (snn_kernels.cu).  CUDA path only; the CPU oracle (oracle/) shares nothing with it.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace snn {

constexpr int kMaxCluster = 16;     // non-portable cluster size limit on B200
constexpr int kMaxThreads = 1024;   // one column per thread -> <= 32 groups of 32 columns per CTA
constexpr int kLutMax = 4096;       // R19
constexpr int kNever = -1;
constexpr int kPadRows = 16;        // fixed-width per-step row slots used by the event engine's block integration

enum : uint32_t { TAG_ENC = 1, TAG_LTD = 2, TAG_LTP = 3, TAG_ROUND = 4, TAG_INIT = 5, TAG_ROUND_LTD = 6 };
enum : int { FLAG_RASTER_INPUT = 1, FLAG_KEEP_STATE = 2, FLAG_RECORD_INPUT = 4, FLAG_ASYNC = 8, FLAG_FLOOR = 16,
             FLAG_NO_LEARN = 64 };   // internal: frozen weights (per-step engine inference, R21)

// Everything one network needs inside the persistent kernel.  Built per launch on the host.
struct Mailbox;

constexpr int kExpDeg = 13;   // degree of the Taylor polynomial of R28's e^y recipe

struct NetDesc {
  // geometry
  int n_in, n_exc, bits, q_max;
  int cs;          // CTAs per network (= cluster size)
  int ngroups;     // ceil(n_exc / 32): columns are sliced across CTAs in groups of 32
  int wpr;         // u32 words per weight row of one CTA slice (max_groups * bits)
  int slice_words; // u32 words of one CTA slice: (n_in + 1) rows (row n_in is all zero), rounded to 4
  int nwi, nwe;    // u32 words per input / output raster row
  // LIF
  int membrane_mode;
  float af, bf, cf, dtf, kI, ief, vthf, vresetf, vinitf;
  long long A, B, C, E;
  int Vth, Vreset, Vinit;
  int t_ref, t_inh, wta_mode, inh_mode, stdp_mode, t_ltp;
  int L_pot, L_dep;
  // 32-bit floating-point conductance (bits = 32, NEXT-2, R28): eqs.(4)(5) parameters, the
  // binary64 e^y recipe's Taylor coefficients 1/m! (host-built, c_m = c_{m-1}/m), I = S * (float)v_spike
  double alpha_p, beta_p, alpha_d, beta_d, g_min, g_max;
  double ecoef[kExpDeg + 1];
  float kV, gminf, gmaxf;
  // tables (device)
  const unsigned long long* thr_enc;   // [256]      event iff u <  thr
  const uint32_t* pot_m1;              // [L_pot]    event iff u <= thr - 1   (thr >= 1 for D < L)
  const uint32_t* dep_m1;              // [L_dep]
  const int* det_base_p;               // [q_max+1]  deterministic arm (R16/R17)
  const uint32_t* det_thr_p;
  const int* det_base_d;
  const uint32_t* det_thr_d;
  // persistent device state
  uint32_t* wslices;                   // [cs][n_in][wpr] packed codes (the smem image of each CTA)
  int* v;                              // [n_exc] fp32 bits or Q15.16
  int* cnt;                            // [n_exc]
  int* last_post;                      // [n_exc]
  int* last_pre;                       // [n_in]
  unsigned long long* stats;           // [8]
  // per-launch I/O
  const uint8_t* images;               // [n_images][n_in]
  const uint32_t* in_raster;           // [T][nwi] with FLAG_RASTER_INPUT (n_images == 1)
  const unsigned long long* seeds;     // [n_images]
  uint32_t* raster_out;                // [T][nwe] output raster of the last image (may be null)
  uint32_t* in_raster_out;             // [T][nwi] input raster of the last image (may be null)
  int* spike_counts;                   // [n_images] (may be null)
  uint32_t* neuron_counts;             // [n_images][n_exc] spikes per neuron and image (FLAG_NO_LEARN; may be null)
  int n_images, T, flags, t0;
  // event engine: per-image active-row lists from the encoder pre-pass
  const uint32_t* ev_offs;             // [n_images][T+1] prefix offsets into ev_rows
  const uint16_t* ev_rows;             // [n_images][rows_stride] active input rows, step-major, ascending
  const uint16_t* ev_rows16;           // [n_images][T][kPadRows] first kPadRows rows of each step, padded with n_in
  long long rows_stride;
  int rows_cap, offs_cap, logn;        // on-chip window of the lists, per-thread LTD undo-log entries
  int floor_epochs;                    // SNN_FLOOR_PROBE on the lean kernel: skeleton epochs per image
  // optional per-epoch trace: [cs][trace_cap][8] u64 (%globaltimer ns)
  unsigned long long* trace;
  int trace_cap;
  // column sharding across ranks: this network is columns [col_base, col_base + n_exc)
  // of a network of n_exc_total; per epoch the rank summaries meet in every rank's mailbox
  int col_base, n_exc_total, world, shard;
  Mailbox* mbox;                  // this rank's mailbox
  Mailbox* const* peers;          // device array [world] of every rank's mailbox (own, peer or IPC pointers)
};

// One rank's mailbox of the column-sharded exchange.  Epochs are numbered by a
// per-shard counter that persists across launches (`seq`, identical on every shard because the
// epoch sequence is).  slot[seq & 1][r] holds rank r's summary of epoch seq as four LL words
// {data32 | seq32 << 32} (W1, count, key hi, key lo): a reader spins until all four carry seq, so
// no fence is needed and a stale word can never pass (slots are rewritten every second epoch).
// flag = max over signals of (seq << 32 | ~step): the earliest crossing step reported for epoch
// seq by another shard (values of older epochs lose the max and are ignored).
constexpr int kMaxWorld = 32;
struct Mailbox {
  unsigned long long slot[2][kMaxWorld][4];
  unsigned long long flag;
  unsigned int seq;               // epochs completed by this shard (written at the end of each launch)
  unsigned int pad[29];
};

struct LaunchParams {
  const NetDesc* descs;   // device array (ensembles) or null -> use `single`
  NetDesc single;
};

// kernels.cu entry points (host side)
cudaError_t launch_present(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, cudaStream_t s);
// event engine (snn_event.cu)
constexpr int kEvMaxThreads = 256;   // 255 registers per thread: the speculation loop keeps all its state in registers
constexpr int kEvMaxT = 32767;
constexpr unsigned long long kShardTimeoutNs = 20000000000ull;   // a missing rank traps after 20 s
size_t event_smem_bytes(int n_in, int slice_words, int L_pot, int L_dep, int q_max, int nthr, int rows_cap,
                        int offs_cap, int logn);
inline int slice_words_for(int n_in, int wpr) { return (((n_in + 1) * wpr) + 3) & ~3; }
cudaError_t query_max_clusters_event(int bits, int cpt, int fixed, int cs, int nthr, size_t smem, int* out);
int event_threads(int max_groups, int bits, int cpt);
cudaError_t launch_encode(const uint8_t* images, const unsigned long long* thr_enc, const unsigned long long* seeds,
                          int n_in, int T, int n_images, int t0, uint32_t* words, uint32_t* counts, cudaStream_t s);
cudaError_t launch_counts_from_raster(const uint32_t* raster, int n_in, int T, uint32_t* counts, cudaStream_t s);
cudaError_t launch_compact(const uint32_t* words, const uint32_t* counts, int n_in, int T, int n_images,
                           long long rows_stride, uint32_t* offs, uint16_t* rows, uint16_t* rows16, cudaStream_t s);
cudaError_t launch_present_event_mode(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, int bits,
                                      int cpt, int fixed, cudaStream_t s);
cudaError_t configure_present_kernel(size_t smem, int cs);
// lean event kernel (snn_lean.cu)
size_t lean_smem_bytes(int n_in, int slice_words, int L_pot, int L_dep, int nthr, int rows_cap, int offs_cap,
                       int logn);
cudaError_t query_max_clusters_lean(int bits, int cpt, int fixed, int cs, int nthr, size_t smem, int* out);
cudaError_t launch_present_lean(const LaunchParams& lp, int n_nets, int cs, int nthr, size_t smem, int bits, int cpt,
                                int fixed, int sharded, int layer, cudaStream_t s);
cudaError_t query_max_clusters(int cs, int nthr, size_t smem, int* out);
cudaError_t launch_init_weights(const NetDesc& d, uint64_t init_seed, cudaStream_t s);
cudaError_t launch_pack_weights(const NetDesc& d, const void* codes, cudaStream_t s);      // u8 / u16 (bits 16) codes
cudaError_t launch_unpack_weights(const NetDesc& d, void* codes, cudaStream_t s);
cudaError_t launch_check_g(const float* g, size_t n, float gmin, float gmax, int* bad, cudaStream_t s);
cudaError_t launch_check_codes(const void* codes, size_t n, int bits, int q_max, int* bad, cudaStream_t s);
size_t present_smem_bytes(int n_in, int wpr, int L_pot, int L_dep, int q_max, int nthr);

// ---- NEXT-1: batch-parallel inference with frozen weights (snn_infer.cu)
constexpr int kMaxClasses = 64;
constexpr int kInferMaxCols = 7 * 32 * 32;   // 224 column threads x 32 columns
struct InferDesc {
  int n_in, n_exc, bits, T, n_images, nwi;
  int nthr_cols;      // column threads: ceil(n_exc / 32)
  int wpr;            // u32 words per weight row of the inference layout (multiple of 4)
  int R, rmax;        // ring slots (power of two) and the largest step served from the ring (R / 2)
  int row_bytes;      // wpr * 4
  float af, bf, cf, dtf, kI, ief, vthf, vresetf, vinitf;
  long long A, B, C, E;
  int Vth, Vreset, Vinit;
  int t_ref, t_inh, wta_mode, inh_mode;
  const uint32_t* w;                 // [n_in][wpr] codes, column j at word j / (32/bits), bits (j % (32/bits)) * bits
  const uint32_t* words;             // [n_images][T][nwi] encoded input spikes
  uint32_t* counts;                  // [n_images][n_exc] spike counts (zeroed by the caller)
  unsigned long long* stats;         // [3] += sum_t act(t), post spikes, LIF column-steps run (may be null)
};
size_t infer_smem_bytes(int R, int row_bytes);
cudaError_t infer_occupancy(int bits, int fixed, int minb, int nthr, size_t smem, int* out);
cudaError_t launch_infer(const InferDesc& d, int grid, int nthr, size_t smem, int fixed, int minb, cudaStream_t s);
cudaError_t launch_pack_infer(const uint8_t* codes, int n_in, int n_exc, int bits, int wpr, uint32_t* w,
                              cudaStream_t s);
cudaError_t launch_label(const uint32_t* counts, int n_images, int n_exc, const int32_t* classes, int n_classes,
                         int32_t* labels, cudaStream_t s);
cudaError_t launch_classify(const uint32_t* counts, int n_images, int n_exc, const int32_t* labels, int n_classes,
                            int32_t* pred, cudaStream_t s);

// ---- NEXT-4: Fig. 4 sparse workload (snn_sparse.cu)
struct SparseDesc {
  int n_in, n_lif, T, n_trials, t_ref;
  float af, bf, cf, dtf, kI, ief, vthf, vresetf, vinitf;
  long long A, B, C, E;
  int Vth, Vreset, Vinit;
  const int32_t* src_off;            // [n_in + n_lif + 1] CSR by source
  const uint16_t* tgt;               // [n_syn] target neuron
  const uint8_t* q;                  // [n_syn] code
  const unsigned long long* thr_enc; // [256]
  const uint8_t* images;             // [n_trials][n_in]
  const unsigned long long* seeds;   // [n_trials]
  uint32_t* counts;                  // [n_trials][n_lif] (zeroed by the caller)
  uint32_t* raster;                  // [n_trials][T][ceil(n_lif/32)] or null (zeroed by the caller)
  unsigned long long* stats;         // [2] += input spikes, neuron spikes
};
constexpr int kSparseMaxLif = 16384;
size_t sparse_smem_bytes(int n_in, int n_lif);
cudaError_t sparse_occupancy(int fixed, int nthr, size_t smem, int* out);
cudaError_t launch_sparse(const SparseDesc& d, int grid, int nthr, size_t smem, int fixed, cudaStream_t s);

}  // namespace snn
