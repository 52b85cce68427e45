// snn_api.cu -- host runtime behind include/snn.h: parameter validation, host-side probability
// tables (built here in double precision, independently of the CPU oracle), device allocation,
// the on-chip layout choice, launches and readout.
#include "snn.h"
#include "snn_internal.h"

#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <string>
#include <vector>
#include <algorithm>

using snn::NetDesc;

namespace {

thread_local std::string g_err;

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

#define CUDA_TRY(expr)                                                                          \
  do {                                                                                          \
    cudaError_t _e = (expr);                                                                    \
    if (_e != cudaSuccess) return fail(SNN_ECUDA, "%s: %s (%s:%d)", #expr, cudaGetErrorString(_e), \
                                       __FILE__, __LINE__);                                     \
  } while (0)

template <class T>
cudaError_t dalloc(T** p, size_t n) {
  *p = nullptr;
  if (n == 0) n = 1;
  return cudaMalloc(reinterpret_cast<void**>(p), n * sizeof(T));
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// threshold of an event of probability P: floor(P * 2^32) (R13)
unsigned long long prob_thr(double P) { return (unsigned long long)std::floor(std::ldexp(P, 32)); }

}  // namespace

struct snn_handle {
  int dev = 0;
  int n_in = 0, n_exc = 0, bits = 0, frac_bits = 0, q_max = 0;
  snn_params p{};
  int cs = 1, nthr = 128, wpr = 0, ngroups = 0, slice_words = 0;
  size_t smem = 0;
  int L_pot = 0, L_dep = 0;
  // fixed / fp32 constants
  long long A = 0, B = 0, C = 0, E = 0;
  int Vth = 0, Vreset = 0, Vinit = 0;
  // device memory
  uint32_t* d_w = nullptr;
  unsigned long long* d_enc = nullptr;
  uint32_t* d_pot = nullptr;
  uint32_t* d_dep = nullptr;
  int* d_dbp = nullptr;
  int* d_dbd = nullptr;
  uint32_t* d_dtp = nullptr;
  uint32_t* d_dtd = nullptr;
  int* d_v = nullptr;
  int* d_cnt = nullptr;
  int* d_lpost = nullptr;
  int* d_lpre = nullptr;
  unsigned long long* d_stats = nullptr;
  uint32_t* d_raster = nullptr;  size_t raster_cap = 0;
  uint32_t* d_inrec = nullptr;   size_t inrec_cap = 0;
  uint8_t* d_img = nullptr;      size_t img_cap = 0;
  uint32_t* d_rin = nullptr;     size_t rin_cap = 0;
  unsigned long long* d_seeds = nullptr; size_t seeds_cap = 0;
  int* d_counts = nullptr;       size_t counts_cap = 0;
  uint8_t* d_codes = nullptr;
  int* d_bad = nullptr;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int last_T = 0;
  bool last_recorded = false;
  int t_next = 0;
  long long launches = 0;
  // snn_set_profile: CUDA events recorded on the handle's stream around every presentation kernel
  bool prof = false;
  std::vector<cudaEvent_t> prof_ev;    // pairs (start, stop)
  size_t prof_used = 0;
  // event engine
  int engine = SNN_ENGINE_EVENT;
  int rows_cap = 0, offs_cap = 0, logn = 0;
  int cpt = 1;                    // columns per thread of the event engine
  bool lean = false;              // event engine runs the lean kernel (HARD / RESET / stochastic)
  size_t smem_lean = 0;
  uint32_t* d_words = nullptr;   size_t words_cap = 0;
  uint32_t* d_ecnt = nullptr;    size_t ecnt_cap = 0;
  uint32_t* d_offs = nullptr;    size_t offs_buf_cap = 0;
  uint16_t* d_rows = nullptr;    size_t rows_buf_cap = 0;
  uint16_t* d_rows16 = nullptr;  size_t rows16_cap = 0;
  unsigned long long* d_trace = nullptr; int trace_epochs = 0;
  int max_clusters = 0;          // co-resident clusters of this launch shape
  // column sharding
  int col_base = 0, n_exc_total = 0, world = 1, shard = 0;
  snn::Mailbox* d_mbox = nullptr;
  snn::Mailbox** d_peers = nullptr;
  std::vector<void*> ipc_opened;       // peer mailboxes opened with cudaIpcOpenMemHandle
  std::vector<snn_handle*> linked;     // in-process shards (snn_shard_link), rank order
  bool connected = false;
  // NEXT-1 inference: weights in the inference layout, rebuilt when w_version moves
  long long w_version = 0, infer_version = -1;
  uint32_t* d_winf = nullptr;     size_t winf_cap = 0;
  uint32_t* d_iwords = nullptr;   size_t iwords_cap = 0;
  uint32_t* d_icounts = nullptr;  size_t icounts_cap = 0;
  uint32_t* d_iecnt = nullptr;    size_t iecnt_cap = 0;
  int32_t* d_cls = nullptr;       size_t cls_cap = 0;
  int32_t* d_lab = nullptr;       size_t lab_cap = 0;
  unsigned long long* d_istats = nullptr;
  unsigned long long* d_iscratch = nullptr;   // per-step engine inference: the kernel's learning-stats slots
  // NEXT-4 sparse workload
  int32_t* d_soff = nullptr;      size_t soff_cap = 0;
  uint16_t* d_stgt = nullptr;     size_t stgt_cap = 0;
  uint8_t* d_sq = nullptr;        size_t sq_cap = 0;
  uint32_t* d_scounts = nullptr;  size_t scounts_cap = 0;
  uint32_t* d_sraster = nullptr;  size_t sraster_cap = 0;
  unsigned long long* d_sstats = nullptr;
};

namespace {

// bytes per code in the readout layout: u8 (<= 8 bits), u16 (16 bits), binary32 G (32 bits, R28)
size_t code_bytes(int bits) { return bits == 32 ? 4 : (bits > 8 ? 2 : 1); }

int validate(int n_in, int n_exc, int bits, const snn_params* p) {
  if (!p) return fail(SNN_EINVAL, "params is NULL");
  if (n_in < 1 || n_in > 8192) return fail(SNN_EINVAL, "n_in=%d outside [1, 8192]", n_in);
  if (n_exc < 1 || n_exc > (1 << 20)) return fail(SNN_EINVAL, "n_exc=%d outside [1, 2^20]", n_exc);
  if (bits != 2 && bits != 4 && bits != 8 && bits != 16 && bits != 32)
    return fail(SNN_EINVAL, "bits=%d not in {2,4,8,16,32}", bits);
  // 32-bit floating-point conductance (R28): the fixed recipe needs an integer sum; truncation and eq.(8)
  // are roundings onto a fixed-point grid (R17), binary32 rounds to nearest
  if (bits == 32 && p->membrane_mode != SNN_MEM_FP32) return fail(SNN_EINVAL, "bits=32 needs membrane_mode fp32 (R28)");
  if (bits == 32 && p->rounding != SNN_ROUND_NEAREST) return fail(SNN_EINVAL, "bits=32 rounds to nearest only (R28)");
  if (!(p->dt_ms > 0.0)) return fail(SNN_EINVAL, "dt_ms must be > 0");
  if (!(p->f_min_hz >= 0.0 && p->f_max_hz >= p->f_min_hz)) return fail(SNN_EINVAL, "need 0 <= f_min <= f_max");
  if (p->f_max_hz * p->dt_ms * 1e-3 > 1.0) return fail(SNN_EINVAL, "f_max * dt > 1 (spike probability > 1)");
  if (!(p->gamma_pot >= 0.0 && p->gamma_pot <= 1.0 && p->gamma_dep >= 0.0 && p->gamma_dep <= 1.0))
    return fail(SNN_EINVAL, "gamma must lie in [0, 1]");
  if (!(p->tau_pot > 0.0 && p->tau_dep > 0.0)) return fail(SNN_EINVAL, "tau must be > 0");
  if (p->t_ref_steps < 0 || p->t_inh_steps < 0 || p->t_ltp_steps < 0) return fail(SNN_EINVAL, "negative step count");
  if (p->wta_mode < 0 || p->wta_mode > 1 || p->inh_mode < 0 || p->inh_mode > 1) return fail(SNN_EINVAL, "bad wta/inh mode");
  if (p->stdp_mode < 0 || p->stdp_mode > 1 || p->rounding < 0 || p->rounding > 2) return fail(SNN_EINVAL, "bad stdp/rounding mode");
  if (p->membrane_mode < 0 || p->membrane_mode > 1) return fail(SNN_EINVAL, "bad membrane_mode");
  if (p->g_min != 0.0 || !(p->g_max > 0.0)) return fail(SNN_EINVAL, "need g_min == 0 and g_max > 0 (R9)");
  if (p->frac_bits < 0 || p->frac_bits > 16) return fail(SNN_EINVAL, "frac_bits outside [0, 16]");
  if (p->init_mode != 0) return fail(SNN_EINVAL, "init_mode must be 0");
  if (p->stdp_mode == 1 && !(p->alpha_p >= 0 && p->alpha_d >= 0 && p->beta_p >= 0 && p->beta_d >= 0))
    return fail(SNN_EINVAL, "alpha/beta must be >= 0");
  if (p->cluster_size < 0 || p->cluster_size > snn::kMaxCluster) return fail(SNN_EINVAL, "cluster_size outside [0, 16]");
  if (p->engine != SNN_ENGINE_EVENT && p->engine != SNN_ENGINE_STEP && p->engine != SNN_ENGINE_EVENT_GENERAL)
    return fail(SNN_EINVAL, "engine must be 0, 1 or 2");
  return SNN_OK;
}

// eqs.(6)(7) tables (R10, R19): u32 (thr - 1) for D < L, where thr = floor(gamma e^{-D dt/tau} 2^32) >= 1
int exp_table(double gamma, double tau, double dt, std::vector<uint32_t>& out) {
  out.clear();
  if (gamma == 0.0) return SNN_OK;
  for (int D = 0; D < snn::kLutMax; ++D) {
    const unsigned long long thr = prob_thr(gamma * std::exp(-((double)D * dt) / tau));
    if (thr == 0) return SNN_OK;
    out.push_back((uint32_t)(thr - 1ull));
  }
  return fail(SNN_EINVAL, "STDP horizon exceeds %d steps (R19): gamma=%g tau=%g", snn::kLutMax, gamma, tau);
}

void fill_static(const snn_handle* h, NetDesc& d) {
  std::memset(&d, 0, sizeof(d));
  const snn_params& p = h->p;
  d.n_in = h->n_in; d.n_exc = h->n_exc; d.bits = h->bits; d.q_max = h->q_max;
  d.cs = h->cs; d.ngroups = h->ngroups; d.wpr = h->wpr; d.slice_words = h->slice_words;
  d.nwi = (h->n_in + 31) / 32; d.nwe = (h->n_exc + 31) / 32;
  d.membrane_mode = p.membrane_mode;
  const double lsb = std::ldexp(1.0, -h->frac_bits);
  d.af = (float)p.a; d.bf = (float)p.b; d.cf = (float)p.c; d.dtf = (float)p.dt_ms;
  d.kI = (float)(p.v_spike * lsb); d.ief = (float)p.i_ext;
  d.vthf = (float)p.v_th; d.vresetf = (float)p.v_reset; d.vinitf = (float)p.v_init;
  d.A = h->A; d.B = h->B; d.C = h->C; d.E = h->E;
  d.Vth = h->Vth; d.Vreset = h->Vreset; d.Vinit = h->Vinit;
  d.t_ref = p.t_ref_steps; d.t_inh = p.t_inh_steps; d.wta_mode = p.wta_mode; d.inh_mode = p.inh_mode;
  d.stdp_mode = p.stdp_mode; d.t_ltp = p.t_ltp_steps;
  d.L_pot = h->L_pot; d.L_dep = h->L_dep;
  d.alpha_p = p.alpha_p; d.beta_p = p.beta_p; d.alpha_d = p.alpha_d; d.beta_d = p.beta_d;
  d.g_min = p.g_min; d.g_max = p.g_max;
  d.ecoef[0] = 1.0;                                   // R28: 1/m! by c_m = c_{m-1} / m (binary64)
  for (int m = 1; m <= snn::kExpDeg; ++m) d.ecoef[m] = d.ecoef[m - 1] / (double)m;
  d.kV = (float)p.v_spike; d.gminf = (float)p.g_min; d.gmaxf = (float)p.g_max;
  d.thr_enc = h->d_enc; d.pot_m1 = h->d_pot; d.dep_m1 = h->d_dep;
  d.det_base_p = h->d_dbp; d.det_thr_p = h->d_dtp; d.det_base_d = h->d_dbd; d.det_thr_d = h->d_dtd;
  d.wslices = h->d_w;
  d.v = h->d_v; d.cnt = h->d_cnt; d.last_post = h->d_lpost; d.last_pre = h->d_lpre;
  d.stats = h->d_stats;
  d.rows_cap = h->rows_cap; d.offs_cap = h->offs_cap; d.logn = h->logn;
  d.trace = h->d_trace; d.trace_cap = h->trace_epochs;
  d.col_base = h->col_base; d.n_exc_total = h->n_exc_total; d.world = 1; d.shard = h->shard;
}

// Sharded launch fields: this rank's mailbox and every rank's.
int shard_arm(snn_handle* h, NetDesc& d) {
  if (h->world <= 1) return SNN_OK;
  if (!h->connected) return fail(SNN_EINVAL, "shard %d of %d is not connected (snn_shard_connect / snn_shard_link)",
                                 h->shard, h->world);
  d.world = h->world; d.shard = h->shard; d.mbox = h->d_mbox; d.peers = h->d_peers;
  return SNN_OK;
}

void free_all(snn_handle* h) {
  for (void* q : h->ipc_opened) if (q) cudaIpcCloseMemHandle(q);
  h->ipc_opened.clear();
  void* ptrs[] = {h->d_w, h->d_enc, h->d_pot, h->d_dep, h->d_dbp, h->d_dbd, h->d_dtp, h->d_dtd,
                  h->d_v, h->d_cnt, h->d_lpost, h->d_lpre, h->d_stats, h->d_raster, h->d_inrec,
                  h->d_img, h->d_rin, h->d_seeds, h->d_counts, h->d_codes, h->d_bad,
                  h->d_words, h->d_ecnt, h->d_offs, h->d_rows, h->d_rows16, h->d_trace,
                  h->d_mbox, h->d_peers, h->d_winf, h->d_iwords, h->d_icounts, h->d_iecnt, h->d_cls,
                  h->d_lab, h->d_istats, h->d_iscratch, h->d_soff, h->d_stgt, h->d_sq, h->d_scounts, h->d_sraster,
                  h->d_sstats};
  for (void* q : ptrs) if (q) cudaFree(q);
  for (cudaEvent_t e : h->prof_ev) cudaEventDestroy(e);
  h->prof_ev.clear();
  if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
}

template <class T>
int ensure(snn_handle* h, T** buf, size_t* cap, size_t need) {
  if (*cap >= need && *buf) return SNN_OK;
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  if (*buf) cudaFree(*buf);
  *buf = nullptr;
  *cap = 0;
  CUDA_TRY(dalloc(buf, need));
  *cap = need;
  return SNN_OK;
}

struct DevGuard {
  int prev = -1;
  explicit DevGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DevGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

// Stage one input array onto the device (returns a device pointer valid on h->stream).
template <class T>
int stage(snn_handle* h, const T* src, size_t n, T** dbuf, size_t* cap, const T** out) {
  if (is_device_ptr(src)) { *out = src; return SNN_OK; }
  int rc = ensure(h, dbuf, cap, n);
  if (rc) return rc;
  CUDA_TRY(cudaMemcpyAsync(*dbuf, src, n * sizeof(T), cudaMemcpyHostToDevice, h->stream));
  *out = *dbuf;
  return SNN_OK;
}

int check_handle(const snn_handle* h) {
  if (!h) return fail(SNN_EINVAL, "handle is NULL");
  return SNN_OK;
}

int finish(snn_handle* h, int flags) {
  CUDA_TRY(cudaGetLastError());
  if (!(flags & SNN_ASYNC)) CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

// Event engine pre-pass: encoder (or the given raster) -> per-step active-row lists.
int event_prepass(snn_handle* h, NetDesc& d, const uint8_t* images, const uint32_t* raster, int n_images, int T,
                  int t0, const unsigned long long* seeds) {
  const int nwi = d.nwi;
  int rc;
  const uint32_t* words = nullptr;
  if ((rc = ensure(h, &h->d_ecnt, &h->ecnt_cap, (size_t)n_images * T))) return rc;
  if (raster) {
    words = raster;
    CUDA_TRY(snn::launch_counts_from_raster(raster, h->n_in, T, h->d_ecnt, h->stream));
  } else {
    if ((rc = ensure(h, &h->d_words, &h->words_cap, (size_t)n_images * T * nwi))) return rc;
    CUDA_TRY(snn::launch_encode(images, h->d_enc, seeds, h->n_in, T, n_images, t0, h->d_words, h->d_ecnt, h->stream));
    words = h->d_words;
    h->launches++;
  }
  const long long stride = ((long long)T * h->n_in + 7) & ~7LL;
  if ((rc = ensure(h, &h->d_offs, &h->offs_buf_cap, (size_t)n_images * (T + 1)))) return rc;
  if ((rc = ensure(h, &h->d_rows, &h->rows_buf_cap, (size_t)n_images * stride))) return rc;
  if ((rc = ensure(h, &h->d_rows16, &h->rows16_cap, (size_t)n_images * T * snn::kPadRows))) return rc;
  CUDA_TRY(snn::launch_compact(words, h->d_ecnt, h->n_in, T, n_images, stride, h->d_offs, h->d_rows, h->d_rows16,
                               h->stream));
  h->launches++;
  d.ev_offs = h->d_offs;
  d.ev_rows = h->d_rows;
  d.ev_rows16 = h->d_rows16;
  d.rows_stride = stride;
  if (d.in_raster_out)
    CUDA_TRY(cudaMemcpyAsync(d.in_raster_out, words + (size_t)(n_images - 1) * T * nwi, (size_t)T * nwi * 4,
                             cudaMemcpyDeviceToDevice, h->stream));
  if (d.raster_out) CUDA_TRY(cudaMemsetAsync(d.raster_out, 0, (size_t)T * d.nwe * 4, h->stream));
  return SNN_OK;
}

// snn_set_profile: record an event on the launching stream (pairs around each presentation kernel)
constexpr size_t kProfMaxEvents = 8192;
void prof_mark(snn_handle* h) {
  if (!h->prof || h->prof_used >= kProfMaxEvents) return;
  if (h->prof_used == h->prof_ev.size()) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) { cudaGetLastError(); h->prof = false; return; }
    h->prof_ev.push_back(e);
  }
  cudaEventRecord(h->prof_ev[h->prof_used++], h->stream);
}

// Common path of every single-handle presentation.
int present_impl(snn_handle* h, const void* input, int n_images, int T, const uint64_t* seeds, int32_t* counts,
                 int flags, int t0) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (n_images < 0 || T < 0 || t0 < 0) return fail(SNN_EINVAL, "negative n_images / T / t0");
  if ((flags & SNN_KEEP_STATE) && n_images > 1) return fail(SNN_EINVAL, "SNN_KEEP_STATE needs n_images == 1");
  if ((flags & SNN_RASTER_INPUT) && n_images > 1) return fail(SNN_EINVAL, "SNN_RASTER_INPUT needs n_images == 1");
  if (!(flags & SNN_KEEP_STATE) && t0 != 0) return fail(SNN_EINVAL, "t0 != 0 requires SNN_KEEP_STATE");
  // continuing may not step back in time: stored timers are < t_next <= t0, so every Dt >= 1 indexes the tables
  if ((flags & SNN_KEEP_STATE) && t0 < h->t_next)
    return fail(SNN_EINVAL, "SNN_KEEP_STATE with t0 = %d before the stored state's next step %d", t0, h->t_next);
  const bool ev = h->engine == SNN_ENGINE_EVENT;
  if (ev && T > snn::kEvMaxT) return fail(SNN_EINVAL, "T=%d exceeds %d for the event engine", T, snn::kEvMaxT);
  if (ev && (flags & SNN_FLOOR_PROBE) && !h->lean)
    return fail(SNN_EINVAL, "SNN_FLOOR_PROBE applies to the per-step engine and the lean event kernel");
  if (n_images == 0) {   // nothing to present (a T == 0 presentation still runs: it resets the state, R5)
    h->last_T = 0;
    return SNN_OK;
  }
  if (!input || !seeds) return fail(SNN_EINVAL, "input / seeds is NULL");
  for (snn_handle* o : h->linked)
    if (o != h && o->dev == h->dev)
      return fail(SNN_EINVAL, "shards linked on one device must be presented together (snn_present_many)");
  DevGuard g(h->dev);
  h->w_version++;                      // STDP may change the codes (inference layout is stale)
  NetDesc d;
  fill_static(h, d);
  d.n_images = n_images; d.T = T; d.flags = flags & 0x17; d.t0 = t0;
  const int nwi = d.nwi, nwe = d.nwe;
  const uint32_t* rin = nullptr;
  const uint8_t* img = nullptr;
  if (flags & SNN_RASTER_INPUT) {
    rc = stage(h, static_cast<const uint32_t*>(input), (size_t)T * nwi, &h->d_rin, &h->rin_cap, &rin);
    if (rc) return rc;
    d.in_raster = rin;
  } else {
    rc = stage(h, static_cast<const uint8_t*>(input), (size_t)n_images * h->n_in, &h->d_img, &h->img_cap, &img);
    if (rc) return rc;
    d.images = img;
  }
  const unsigned long long* sd = nullptr;
  rc = stage(h, reinterpret_cast<const unsigned long long*>(seeds), (size_t)n_images, &h->d_seeds, &h->seeds_cap, &sd);
  if (rc) return rc;
  d.seeds = sd;
  rc = ensure(h, &h->d_raster, &h->raster_cap, (size_t)T * nwe);
  if (rc) return rc;
  d.raster_out = h->d_raster;
  if (flags & SNN_RECORD_INPUT) {
    rc = ensure(h, &h->d_inrec, &h->inrec_cap, (size_t)T * nwi);
    if (rc) return rc;
    d.in_raster_out = h->d_inrec;
  }
  const bool counts_dev = counts && is_device_ptr(counts);
  if (counts && !counts_dev) {
    rc = ensure(h, &h->d_counts, &h->counts_cap, (size_t)n_images);
    if (rc) return rc;
    d.spike_counts = h->d_counts;
  } else {
    d.spike_counts = counts;
  }
  snn::LaunchParams lp;
  lp.descs = nullptr;
  if (ev) {
    rc = event_prepass(h, d, img, rin, n_images, T, (flags & SNN_KEEP_STATE) ? t0 : 0, sd);
    if (rc) return rc;
    if ((rc = shard_arm(h, d))) return rc;
    if (flags & SNN_FLOOR_PROBE) {       // the handle's mean epochs per image so far (stats [8] / [6])
      unsigned long long st[SNN_NSTATS];
      CUDA_TRY(cudaMemcpyAsync(st, h->d_stats, sizeof(st), cudaMemcpyDeviceToHost, h->stream));
      CUDA_TRY(cudaStreamSynchronize(h->stream));
      if (st[6] == 0) return fail(SNN_EINVAL, "SNN_FLOOR_PROBE needs learning presentations first (epochs per image)");
      d.floor_epochs = (int)((st[8] + st[6] / 2) / st[6]);
    }
    lp.single = d;
    prof_mark(h);
    if (h->lean)
      CUDA_TRY(snn::launch_present_lean(lp, 1, h->cs, h->nthr, h->smem_lean, h->bits, h->cpt, h->p.membrane_mode,
                                        h->world > 1, h->p.wta_mode == SNN_WTA_LAYER, h->stream));
    else
      CUDA_TRY(snn::launch_present_event_mode(lp, 1, h->cs, h->nthr, h->smem, h->bits, h->cpt, h->p.membrane_mode,
                                              h->stream));
    prof_mark(h);
  } else {
    if ((rc = shard_arm(h, d))) return rc;
    lp.single = d;
    prof_mark(h);
    CUDA_TRY(snn::launch_present(lp, 1, h->cs, h->nthr, h->smem, h->stream));
    prof_mark(h);
  }
  h->launches++;
  if (counts && !counts_dev)
    CUDA_TRY(cudaMemcpyAsync(counts, h->d_counts, sizeof(int32_t) * n_images, cudaMemcpyDeviceToHost, h->stream));
  h->last_T = T;
  h->last_recorded = (flags & SNN_RECORD_INPUT) != 0;
  h->t_next = ((flags & SNN_KEEP_STATE) ? t0 : 0) + T;
  return finish(h, flags);
}

}  // namespace

extern "C" {

const char* snn_last_error(void) { return g_err.c_str(); }

int snn_params_preset(snn_params* p, int preset) {
  if (!p) return fail(SNN_EINVAL, "params is NULL");
  std::memset(p, 0, sizeof(*p));
  // P:90 §III-D
  p->a = -6.77; p->b = -0.0989; p->c = 0.314; p->v_th = -60.2; p->v_reset = -74.7; p->v_init = -70.0;
  p->dt_ms = 1.0; p->v_spike = 2.0; p->i_ext = 0.0;          // R1, R3
  p->t_ref_steps = 5; p->t_inh_steps = 10;                     // R6, R7
  p->wta_mode = SNN_WTA_HARD; p->inh_mode = SNN_INH_RESET;
  p->stdp_mode = SNN_STDP_STOCH; p->rounding = SNN_ROUND_NEAREST; p->t_ltp_steps = 20;
  p->membrane_mode = SNN_MEM_FP32;
  // Table I "16 bit" row alpha/beta (R16) for the deterministic arm at every width
  p->alpha_p = 0.01; p->beta_p = 3.0; p->alpha_d = 0.005; p->beta_d = 3.0; p->g_min = 0.0; p->g_max = 1.0;
  p->frac_bits = 0; p->init_mode = 0; p->init_seed = 1; p->cluster_size = 0;
  p->f_min_hz = 1.0; p->f_max_hz = 22.0;
  switch (preset) {   // Table I
    case SNN_PRESET_2B:  p->gamma_pot = 0.2; p->tau_pot = 20; p->gamma_dep = 0.2; p->tau_dep = 10; break;
    case SNN_PRESET_4B:  p->gamma_pot = 0.3; p->tau_pot = 30; p->gamma_dep = 0.3; p->tau_dep = 10; break;
    case SNN_PRESET_8B:  p->gamma_pot = 0.5; p->tau_pot = 30; p->gamma_dep = 0.5; p->tau_dep = 10; break;
    case SNN_PRESET_16B: p->gamma_pot = 0.9; p->tau_pot = 30; p->gamma_dep = 0.9; p->tau_dep = 10; break;
    case SNN_PRESET_HF:
      p->gamma_pot = 0.3; p->tau_pot = 80; p->gamma_dep = 0.2; p->tau_dep = 5;
      p->f_min_hz = 5.0; p->f_max_hz = 78.0;
      break;
    default: return fail(SNN_EINVAL, "unknown preset %d", preset);
  }
  return SNN_OK;
}

}  // extern "C"

namespace {
// A network of columns [col_base, col_base + n_exc) of an n_exc_total-column network (col_base = 0,
// n_exc_total = n_exc: an unsharded network).
// Shards choose their launch shape from the largest shard's column groups (layout_groups) with at most
// as many CTAs as the smallest shard has groups (cs_cap), so every shard of a world has the same
// cluster size, CTA shape and shared-memory plan (one snn_present_many launch can hold them all).
int create_impl(int n_in, int n_exc, int bits, const snn_params* p, int col_base, int n_exc_total, int shard,
                int world, int layout_groups, int cs_cap, snn_handle** out) {
  snn_handle* h = new (std::nothrow) snn_handle();
  if (!h) return fail(SNN_ENOMEM, "host allocation failed");
  int rc;
  h->p = *p;
  h->n_in = n_in; h->n_exc = n_exc; h->bits = bits;
  h->col_base = col_base; h->n_exc_total = n_exc_total; h->shard = shard; h->world = world;
  h->frac_bits = p->frac_bits > 0 ? p->frac_bits : bits;
  h->q_max = bits == 32 ? 0 : (1 << bits) - 1;      // 32 bits: binary32 conductance, no code grid (R28)
  if (bits <= 16 && h->frac_bits != bits) {
    const double cap = std::floor(std::ldexp(p->g_max, h->frac_bits));
    if (cap < h->q_max) h->q_max = (int)cap;
  }
  const double lsb = std::ldexp(1.0, -h->frac_bits);

  // ---- host tables, built in double precision
  unsigned long long enc[256];
  for (int x = 0; x < 256; ++x)
    enc[x] = prob_thr((p->f_min_hz + (p->f_max_hz - p->f_min_hz) * (double)x / 255.0) * p->dt_ms * 1e-3);
  std::vector<uint32_t> pot, dep;
  if ((rc = exp_table(p->gamma_pot, p->tau_pot, p->dt_ms, pot)) || (rc = exp_table(p->gamma_dep, p->tau_dep, p->dt_ms, dep))) {
    delete h;
    return rc;
  }
  h->L_pot = (int)pot.size();
  h->L_dep = (int)dep.size();
  std::vector<int> dbp(h->q_max + 1), dbd(h->q_max + 1);
  std::vector<uint32_t> dtp(h->q_max + 1), dtd(h->q_max + 1);
  for (int q = 0; q <= h->q_max; ++q) {     // eqs.(4)(5) in LSB units, R16/R17
    const double G = (double)q * lsb;
    const double x_p = std::ldexp(p->alpha_p * std::exp(-p->beta_p * (G - p->g_min) / (p->g_max - p->g_min)), h->frac_bits);
    const double x_d = std::ldexp(p->alpha_d * std::exp(-p->beta_d * (p->g_max - G) / (p->g_max - p->g_min)), h->frac_bits);
    for (int s = 0; s < 2; ++s) {
      const double x = s == 0 ? x_p : x_d;
      double base;
      unsigned long long thr = 0;
      if (p->rounding == SNN_ROUND_TRUNC) base = std::floor(x);
      else if (p->rounding == SNN_ROUND_NEAREST) base = std::floor(x + 0.5);
      else { base = std::floor(x); thr = prob_thr(x - std::floor(x)); }
      const int bi = base > 1e9 ? 1000000000 : (int)base;
      if (s == 0) { dbp[q] = bi; dtp[q] = (uint32_t)thr; } else { dbd[q] = bi; dtd[q] = (uint32_t)thr; }
    }
  }
  h->A = std::llround(p->dt_ms * p->a * 65536.0);
  h->B = std::llround(p->dt_ms * p->b * 4294967296.0);
  h->C = std::llround(p->dt_ms * p->c * p->v_spike * lsb * 4294967296.0);
  h->E = std::llround(p->dt_ms * p->c * p->i_ext * 65536.0);
  h->Vth = (int)std::llround(p->v_th * 65536.0);
  h->Vreset = (int)std::llround(p->v_reset * 65536.0);
  h->Vinit = (int)std::llround(p->v_init * 65536.0);

  // ---- device + on-chip layout
  int ndev = 0;
  cudaError_t ce = cudaGetDeviceCount(&ndev);
  if (ce != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    delete h;
    return fail(SNN_ECUDA, "no CUDA device: %s", cudaGetErrorString(ce));
  }
  cudaGetDevice(&h->dev);
  int smem_optin = 0;
  cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, h->dev);
  h->ngroups = (n_exc + 31) / 32;
  // 16-bit codes (NEXT-2, R27) and binary32 conductances (R28) run on the per-step engine: the event kernels
  // pack <= 8-bit codes in SWAR lanes
  h->engine = (p->engine == SNN_ENGINE_STEP || bits > 8) ? SNN_ENGINE_STEP : SNN_ENGINE_EVENT;
  // the lean kernel covers the paper's default learning mode; SNN_NO_LEAN=1 disables it
  // (LAYER WTA is instantiated unsharded only)
  const bool lean_mode = p->engine == SNN_ENGINE_EVENT && bits <= 8 &&
                         (p->wta_mode == SNN_WTA_HARD || (p->wta_mode == SNN_WTA_LAYER && world == 1)) &&
                         p->inh_mode == SNN_INH_RESET && p->stdp_mode == SNN_STDP_STOCH &&
                         !(getenv("SNN_NO_LEAN") && atoi(getenv("SNN_NO_LEAN")) != 0);
  int chosen = 0;
  const bool ev = h->engine == SNN_ENGINE_EVENT;
  const int max_thr = ev ? snn::kEvMaxThreads : snn::kMaxThreads;
  const int cs_lo = p->cluster_size > 0 ? p->cluster_size : 1;
  const int cs_hi = p->cluster_size > 0 ? p->cluster_size : snn::kMaxCluster;
  // event engine: the largest cluster that fits (one exchange per epoch, so more SMs per network win);
  // per-step engine: the smallest (one exchange per step, cheaper with fewer CTAs)
  std::vector<int> order;
  for (int cs = cs_lo; cs <= cs_hi; ++cs) order.push_back(cs);
  if (ev && p->cluster_size == 0) std::reverse(order.begin(), order.end());
  for (int cs : order) {
    if (cs > cs_cap) continue;
    const int max_groups = (layout_groups + cs - 1) / cs;
    // columns per thread: 2 at 2 bits when the CTA stays <= 256 threads (measured best on C4 with
    // tools/sweep.py), else the SWAR maximum 8/bits; SNN_CPT overrides
    int cpt = 1;
    if (ev) {
      const char* env = getenv("SNN_CPT");
      const int cap = 8 / bits;
      cpt = (bits == 2 && snn::event_threads(max_groups, bits, 2) <= max_thr) ? 2 : cap;
      if (env && atoi(env) >= 1 && atoi(env) <= cap && (cap % atoi(env)) == 0) cpt = atoi(env);
    }
    const int nthr = ev ? snn::event_threads(max_groups, bits, cpt) : (max_groups * 32 < 128 ? 128 : max_groups * 32);
    if ((ev ? nthr : max_groups * 32) > max_thr) continue;
    const int wpr = max_groups * bits;
    const int sw = snn::slice_words_for(n_in, wpr);
    size_t smem;
    int rows_cap = 0, offs_cap = 0, logn = 0;
    if (ev) {
      // on-chip window of active-row lists + LTD undo log: shrink until it fits
      const int plans[4][3] = {{std::max(n_in, 4096), 512, 16}, {n_in, 256, 16}, {n_in, 128, 8}, {n_in, 64, 4}};
      // (the lean kernel, when the mode allows it, needs more: prefer the largest window that fits both)
      smem = 0;
      int k_ev = -1, k_lean = -1;
      for (int k = 0; k < 4; ++k) {
        const int lg = p->stdp_mode == SNN_STDP_STOCH ? plans[k][2] : 1;
        const size_t se = snn::event_smem_bytes(n_in, sw, h->L_pot, h->L_dep, h->q_max, nthr, plans[k][0], plans[k][1], lg);
        if (se > (size_t)smem_optin) continue;
        if (k_ev < 0) k_ev = k;
        if (lean_mode && k_lean < 0 &&
            snn::lean_smem_bytes(n_in, sw, h->L_pot, h->L_dep, nthr, plans[k][0], plans[k][1], lg) <= (size_t)smem_optin)
          k_lean = k;
      }
      const int kp = k_lean >= 0 ? k_lean : (k_ev >= 0 ? k_ev : 3);
      rows_cap = plans[kp][0]; offs_cap = plans[kp][1];
      logn = p->stdp_mode == SNN_STDP_STOCH ? plans[kp][2] : 1;
      smem = snn::event_smem_bytes(n_in, sw, h->L_pot, h->L_dep, h->q_max, nthr, rows_cap, offs_cap, logn);
    } else {
      smem = snn::present_smem_bytes(n_in, sw, h->L_pot, h->L_dep, h->q_max, nthr);
    }
    if (smem > (size_t)smem_optin) continue;
    h->cs = cs; h->nthr = nthr; h->wpr = wpr; h->slice_words = sw; h->smem = smem;
    h->rows_cap = rows_cap; h->offs_cap = offs_cap; h->logn = logn; h->cpt = cpt;
    if (ev && lean_mode) {
      h->smem_lean = snn::lean_smem_bytes(n_in, sw, h->L_pot, h->L_dep, nthr, rows_cap, offs_cap, logn);
      h->lean = h->smem_lean <= (size_t)smem_optin;
    }
    chosen = 1;
    break;
  }
  if (!chosen) {
    delete h;
    return fail(SNN_ESIZE, "network %dx%d at %d bits does not fit one cluster of <= 16 CTAs (%d B smem/CTA)",
                n_in, n_exc, bits, smem_optin);
  }
  int nclusters = 0;
  ce = ev ? snn::query_max_clusters_event(bits, h->cpt, p->membrane_mode, h->cs, h->nthr, h->smem, &nclusters)
          : snn::query_max_clusters(h->cs, h->nthr, h->smem, &nclusters);
  if (ce != cudaSuccess || nclusters < 1) {
    cudaGetLastError();
    delete h;
    return fail(SNN_ECOOP, "cluster of %d CTAs x %zu B smem cannot be co-resident (%s)", h->cs, h->smem,
                cudaGetErrorString(ce));
  }
  if (h->cs == 1) {                    // the query returned CTAs per SM
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->dev);
    nclusters *= sms;
  }
  h->max_clusters = nclusters;
  if (h->lean) {
    int nl = 0;
    ce = snn::query_max_clusters_lean(bits, h->cpt, p->membrane_mode, h->cs, h->nthr, h->smem_lean, &nl);
    if (ce != cudaSuccess || nl < 1) { cudaGetLastError(); h->lean = false; }
  }

#define ALLOC(ptr, n)                                                            \
  do {                                                                           \
    if (dalloc(&(ptr), (n)) != cudaSuccess) {                                    \
      cudaGetLastError();                                                        \
      free_all(h);                                                               \
      delete h;                                                                  \
      return fail(SNN_ENOMEM, "cudaMalloc failed for " #ptr);                    \
    }                                                                            \
  } while (0)
  ALLOC(h->d_w, (size_t)h->cs * h->slice_words);
  ALLOC(h->d_enc, 256);
  ALLOC(h->d_pot, pot.size());
  ALLOC(h->d_dep, dep.size());
  ALLOC(h->d_dbp, (size_t)h->q_max + 1);
  ALLOC(h->d_dbd, (size_t)h->q_max + 1);
  ALLOC(h->d_dtp, (size_t)h->q_max + 1);
  ALLOC(h->d_dtd, (size_t)h->q_max + 1);
  ALLOC(h->d_v, (size_t)n_exc);
  ALLOC(h->d_cnt, (size_t)n_exc);
  ALLOC(h->d_lpost, (size_t)n_exc);
  ALLOC(h->d_lpre, (size_t)n_in);
  ALLOC(h->d_stats, SNN_NSTATS);
  ALLOC(h->d_codes, (size_t)n_in * n_exc * code_bytes(bits));
  ALLOC(h->d_bad, 1);
  if (world > 1) {
    ALLOC(h->d_mbox, 1);
    ALLOC(h->d_peers, (size_t)world);
  }
#undef ALLOC
  if (cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking) != cudaSuccess) {
    free_all(h);
    delete h;
    return fail(SNN_ECUDA, "cudaStreamCreate failed");
  }
  h->own_stream = true;
  auto up = [&](void* dst, const void* src, size_t bytes) {
    return bytes ? cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, h->stream) : cudaSuccess;
  };
  cudaError_t e = cudaSuccess;
  if (e == cudaSuccess) e = up(h->d_enc, enc, sizeof(enc));
  if (e == cudaSuccess) e = up(h->d_pot, pot.data(), pot.size() * 4);
  if (e == cudaSuccess) e = up(h->d_dep, dep.data(), dep.size() * 4);
  if (e == cudaSuccess) e = up(h->d_dbp, dbp.data(), dbp.size() * 4);
  if (e == cudaSuccess) e = up(h->d_dbd, dbd.data(), dbd.size() * 4);
  if (e == cudaSuccess) e = up(h->d_dtp, dtp.data(), dtp.size() * 4);
  if (e == cudaSuccess) e = up(h->d_dtd, dtd.data(), dtd.size() * 4);
  // state after a reset (R5)
  std::vector<int> v0(n_exc), m1(std::max(n_in, n_exc), snn::kNever);
  if (p->membrane_mode == SNN_MEM_FIXED) std::fill(v0.begin(), v0.end(), h->Vinit);
  else { float f = (float)p->v_init; int bitsf; std::memcpy(&bitsf, &f, 4); std::fill(v0.begin(), v0.end(), bitsf); }
  if (e == cudaSuccess) e = up(h->d_v, v0.data(), (size_t)n_exc * 4);
  if (e == cudaSuccess) e = cudaMemsetAsync(h->d_cnt, 0, (size_t)n_exc * 4, h->stream);
  if (e == cudaSuccess) e = up(h->d_lpost, m1.data(), (size_t)n_exc * 4);
  if (e == cudaSuccess) e = up(h->d_lpre, m1.data(), (size_t)n_in * 4);
  if (e == cudaSuccess) e = cudaMemsetAsync(h->d_stats, 0, SNN_NSTATS * sizeof(unsigned long long), h->stream);
  if (e == cudaSuccess && h->d_mbox) e = cudaMemsetAsync(h->d_mbox, 0, sizeof(snn::Mailbox), h->stream);
  NetDesc d;
  fill_static(h, d);
  if (e == cudaSuccess) e = snn::launch_init_weights(d, p->init_seed, h->stream);   // R4
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e != cudaSuccess) {
    free_all(h);
    delete h;
    return fail(SNN_ECUDA, "create: %s", cudaGetErrorString(e));
  }
  h->launches = 1;
  *out = h;
  return SNN_OK;
}
}  // namespace

extern "C" {

int snn_create(int n_in, int n_exc, int bits, const snn_params* p, snn_handle** out) {
  if (!out) return fail(SNN_EINVAL, "out is NULL");
  *out = nullptr;
  int rc = validate(n_in, n_exc, bits, p);
  if (rc) return rc;
  const int G = (n_exc + 31) / 32;
  return create_impl(n_in, n_exc, bits, p, 0, n_exc, 0, 1, G, G, out);
}

int snn_create_shard(int n_in, int n_exc_total, int bits, const snn_params* p, int shard, int world,
                     snn_handle** out) {
  if (!out) return fail(SNN_EINVAL, "out is NULL");
  *out = nullptr;
  int rc = validate(n_in, n_exc_total, bits, p);
  if (rc) return rc;
  if (world < 1 || world > snn::kMaxWorld) return fail(SNN_EINVAL, "world=%d outside [1, %d]", world, snn::kMaxWorld);
  if (shard < 0 || shard >= world) return fail(SNN_EINVAL, "shard=%d outside [0, %d)", shard, world);
  // <= 8-bit codes shard on the event engines (one exchange per post-spike epoch), 16-bit codes and binary32
  // conductances on the per-step engine (one exchange per step): a 784 -> 6400 network at 16 / 32 bits spreads
  // over 4 / 8 clusters
  if (p->engine == SNN_ENGINE_EVENT_GENERAL && bits > 8) return fail(SNN_EINVAL, "bits > 8 run on the per-step engine");
  const int G = (n_exc_total + 31) / 32;
  if (G < world) return fail(SNN_EINVAL, "%d column groups of 32 cannot feed %d shards", G, world);
  const int lo = 32 * (int)(((long long)shard * G) / world);
  const int hi = std::min(n_exc_total, 32 * (int)(((long long)(shard + 1) * G) / world));
  return create_impl(n_in, hi - lo, bits, p, lo, n_exc_total, shard, world, (G + world - 1) / world, G / world, out);
}

int snn_shard_ipc_handle(snn_handle* h, void* out, size_t cap) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (h->world <= 1 || !h->d_mbox) return fail(SNN_EINVAL, "not a shard of a world > 1");
  if (!out || cap < SNN_IPC_HANDLE_BYTES) return fail(SNN_ESIZE, "need %d bytes", SNN_IPC_HANDLE_BYTES);
  static_assert(sizeof(cudaIpcMemHandle_t) == SNN_IPC_HANDLE_BYTES, "IPC handle size");
  DevGuard g(h->dev);
  cudaIpcMemHandle_t ih;
  CUDA_TRY(cudaIpcGetMemHandle(&ih, h->d_mbox));
  std::memcpy(out, &ih, sizeof(ih));
  return SNN_OK;
}

int snn_shard_connect(snn_handle* h, const void* handles, size_t n_bytes) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (h->world <= 1 || !h->d_mbox) return fail(SNN_EINVAL, "not a shard of a world > 1");
  if (h->connected) return fail(SNN_EINVAL, "shard already connected");
  if (!handles || n_bytes < (size_t)h->world * SNN_IPC_HANDLE_BYTES)
    return fail(SNN_ESIZE, "need world x %d handle bytes", SNN_IPC_HANDLE_BYTES);
  DevGuard g(h->dev);
  std::vector<snn::Mailbox*> peers(h->world, nullptr);
  for (int r = 0; r < h->world; ++r) {
    if (r == h->shard) { peers[r] = h->d_mbox; continue; }
    cudaIpcMemHandle_t ih;
    std::memcpy(&ih, static_cast<const char*>(handles) + (size_t)r * SNN_IPC_HANDLE_BYTES, sizeof(ih));
    void* ptr = nullptr;
    const cudaError_t e = cudaIpcOpenMemHandle(&ptr, ih, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      cudaGetLastError();
      for (void* q : h->ipc_opened) cudaIpcCloseMemHandle(q);
      h->ipc_opened.clear();
      return fail(SNN_ECUDA, "opening the mailbox of shard %d: %s", r, cudaGetErrorString(e));
    }
    h->ipc_opened.push_back(ptr);
    peers[r] = static_cast<snn::Mailbox*>(ptr);
  }
  CUDA_TRY(cudaMemcpy(h->d_peers, peers.data(), sizeof(void*) * h->world, cudaMemcpyHostToDevice));
  h->connected = true;
  return SNN_OK;
}

int snn_shard_link(snn_handle* const* hs, int world) {
  if (!hs || world < 2) return fail(SNN_EINVAL, "need >= 2 shard handles");
  for (int r = 0; r < world; ++r) {
    const snn_handle* h = hs[r];
    if (!h) return fail(SNN_EINVAL, "handle %d is NULL", r);
    if (h->world != world || h->shard != r) return fail(SNN_EINVAL, "hs[%d] is not shard %d of %d", r, r, world);
    if (h->connected) return fail(SNN_EINVAL, "shard %d already connected", r);
    if (h->n_in != hs[0]->n_in || h->n_exc_total != hs[0]->n_exc_total || h->bits != hs[0]->bits)
      return fail(SNN_EINVAL, "shards of one network must share n_in, n_exc_total, bits");
  }
  std::vector<snn::Mailbox*> peers(world);
  for (int r = 0; r < world; ++r) peers[r] = hs[r]->d_mbox;
  for (int r = 0; r < world; ++r) {
    snn_handle* h = hs[r];
    DevGuard g(h->dev);
    for (int o = 0; o < world; ++o) {
      if (hs[o]->dev == h->dev) continue;
      int ok = 0;
      CUDA_TRY(cudaDeviceCanAccessPeer(&ok, h->dev, hs[o]->dev));
      if (!ok) return fail(SNN_ECUDA, "device %d cannot access device %d", h->dev, hs[o]->dev);
      const cudaError_t e = cudaDeviceEnablePeerAccess(hs[o]->dev, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return fail(SNN_ECUDA, "%s", cudaGetErrorString(e));
      cudaGetLastError();
    }
    CUDA_TRY(cudaMemcpy(h->d_peers, peers.data(), sizeof(void*) * world, cudaMemcpyHostToDevice));
  }
  for (int r = 0; r < world; ++r) {
    hs[r]->linked.assign(hs, hs + world);
    hs[r]->connected = true;
  }
  return SNN_OK;
}

int snn_destroy(snn_handle* h) {
  if (!h) return SNN_OK;
  DevGuard g(h->dev);
  if (h->stream) cudaStreamSynchronize(h->stream);
  for (snn_handle* o : h->linked)      // the rest of its world can no longer run
    if (o != h) { o->linked.clear(); o->connected = false; }
  free_all(h);
  delete h;
  return SNN_OK;
}

int snn_set_stream(snn_handle* h, void* s) {
  int rc = check_handle(h);
  if (rc) return rc;
  DevGuard g(h->dev);
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  if (s) {
    if (h->own_stream) cudaStreamDestroy(h->stream);
    h->stream = static_cast<cudaStream_t>(s);
    h->own_stream = false;
  } else if (!h->own_stream) {
    CUDA_TRY(cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking));
    h->own_stream = true;
  }
  return SNN_OK;
}

int snn_synchronize(snn_handle* h) {
  int rc = check_handle(h);
  if (rc) return rc;
  DevGuard g(h->dev);
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_present(snn_handle* h, const uint8_t* image, int T, uint64_t seed) {
  return present_impl(h, image, 1, T, &seed, nullptr, 0, 0);
}

int snn_present_ex(snn_handle* h, const void* input, int T, uint64_t seed, int flags, int t0) {
  if (flags & SNN_ASYNC) return fail(SNN_EINVAL, "snn_present_ex is synchronous (seed is passed by value)");
  return present_impl(h, input, 1, T, &seed, nullptr, flags, t0);
}

int snn_present_raster(snn_handle* h, const uint32_t* raster, int T, uint64_t seed) {
  return present_impl(h, raster, 1, T, &seed, nullptr, SNN_RASTER_INPUT, 0);
}

int snn_present_batch(snn_handle* h, const uint8_t* images, int n_images, int T, const uint64_t* seeds,
                      int32_t* spike_counts, int flags) {
  if (flags & (SNN_RASTER_INPUT | SNN_KEEP_STATE)) return fail(SNN_EINVAL, "batch presentations take images, fresh state");
  // SNN_FLOOR_PROBE (16): benchmark-only probe of the per-step synchronisation floor (no learning work)
  return present_impl(h, images, n_images, T, seeds, spike_counts, flags, 0);
}

}  // extern "C"

namespace {
// One launch for n handles (ensembles, linked shards).  kflags = FLAG_NO_LEARN (per-step engine only): inference,
// spike counts per neuron and image into ncounts[k] (device buffers), the handles' weights and state untouched.
int present_many_impl(snn_handle* const* hs, int n, const uint8_t* const* images, int n_images, int T,
                      const uint64_t* const* seeds, int kflags, uint32_t* const* ncounts) {
  if (!hs || n < 1 || !images || !seeds) return fail(SNN_EINVAL, "bad ensemble arguments");
  const bool infer = (kflags & snn::FLAG_NO_LEARN) != 0;
  if (n_images < 0 || T < 0) return fail(SNN_EINVAL, "negative n_images / T");
  for (int k = 0; k < n; ++k) {
    if (!hs[k]) return fail(SNN_EINVAL, "handle %d is NULL", k);
    const bool same_shape = hs[k]->engine == SNN_ENGINE_EVENT ? (hs[k]->bits != hs[0]->bits || hs[k]->nthr == hs[0]->nthr)
                                                              : hs[k]->nthr == hs[0]->nthr;
    if (hs[k]->n_in != hs[0]->n_in || hs[k]->cs != hs[0]->cs || !same_shape ||
        hs[k]->dev != hs[0]->dev || hs[k]->engine != hs[0]->engine ||
        hs[k]->p.membrane_mode != hs[0]->p.membrane_mode)
      return fail(SNN_EINVAL, "ensemble handles must share n_in, cluster size, CTA shape, engine, membrane mode, device");
    for (int m = 0; m < k; ++m)
      if (hs[m] == hs[k]) return fail(SNN_EINVAL, "handle %d appears twice", k);
    if (infer && hs[k]->engine != SNN_ENGINE_STEP)
      return fail(SNN_EINVAL, "snn_infer_many runs per-step-engine handles (bits 16 / 32 or SNN_ENGINE_STEP)");
    if (!infer) hs[k]->w_version++;
    if (hs[k]->world > 1) {        // every shard of its world must be in this launch (they wait on each other)
      if (hs[k]->linked.empty()) return fail(SNN_EINVAL, "shard handle %d is not linked in this process", k);
      for (snn_handle* o : hs[k]->linked)
        if (std::find(hs, hs + n, o) == hs + n) return fail(SNN_EINVAL, "handle %d: its world is incomplete", k);
    }
  }
  {
    int nsh = 0;
    for (int k = 0; k < n; ++k) nsh += hs[k]->world > 1 ? 1 : 0;
    if (nsh > 0 && n > hs[0]->max_clusters)
      return fail(SNN_ECOOP, "%d networks cannot be co-resident (%d clusters fit)", n, hs[0]->max_clusters);
  }
  const bool ev = hs[0]->engine == SNN_ENGINE_EVENT;
  if (ev && T > snn::kEvMaxT) return fail(SNN_EINVAL, "T=%d exceeds %d for the event engine", T, snn::kEvMaxT);
  if (n_images == 0) return SNN_OK;
  snn_handle* h0 = hs[0];
  DevGuard g(h0->dev);
  std::vector<NetDesc> descs(n);
  for (int k = 0; k < n; ++k) {
    snn_handle* h = hs[k];
    if (h != h0) CUDA_TRY(cudaStreamSynchronize(h->stream));
    cudaStream_t own = h->stream;
    h->stream = h0->stream;            // all pre-pass work is ordered on the launching stream
    NetDesc& d = descs[k];
    fill_static(h, d);
    d.n_images = n_images; d.T = T; d.flags = kflags; d.t0 = 0;
    if (infer) {                       // inference: the learning counters are left alone (scratch slots)
      if (!h->d_iscratch && dalloc(&h->d_iscratch, SNN_NSTATS) != cudaSuccess) {
        cudaGetLastError();
        h->stream = own;
        return fail(SNN_ENOMEM, "scratch allocation failed");
      }
      cudaMemsetAsync(h->d_iscratch, 0, SNN_NSTATS * sizeof(unsigned long long), h0->stream);
      d.stats = h->d_iscratch;
      d.neuron_counts = ncounts[k];
    }
    const uint8_t* img = nullptr;
    const unsigned long long* sd = nullptr;
    int rc = stage(h, images[k], (size_t)n_images * h->n_in, &h->d_img, &h->img_cap, &img);
    if (!rc) rc = stage(h, reinterpret_cast<const unsigned long long*>(seeds[k]), (size_t)n_images, &h->d_seeds,
                        &h->seeds_cap, &sd);
    if (!rc) rc = ensure(h, &h->d_raster, &h->raster_cap, (size_t)T * d.nwe);
    if (!rc) {
      d.images = img; d.seeds = sd; d.raster_out = infer ? nullptr : h->d_raster;
      if (ev) rc = event_prepass(h, d, img, nullptr, n_images, T, 0, sd);
      if (!rc) rc = shard_arm(h, d);
    }
    h->stream = own;
    if (rc) return rc;
  }
  // event engine: one launch per bit width (the kernel is specialised on it), the groups run
  // concurrently on forked streams; step engine: one launch for the whole ensemble.
  std::vector<std::vector<int>> groups;
  if (ev) {
    for (int bw : {2, 4, 8}) {
      std::vector<int> g;
      for (int k = 0; k < n; ++k) if (hs[k]->bits == bw) g.push_back(k);
      if (!g.empty()) groups.push_back(g);
    }
  } else {
    std::vector<int> g;
    for (int k = 0; k < n; ++k) g.push_back(k);
    groups.push_back(g);
  }
  NetDesc* d_descs = nullptr;
  CUDA_TRY(cudaMalloc(&d_descs, sizeof(NetDesc) * n));
  std::vector<NetDesc> ordered;
  for (auto& g : groups) for (int k : g) ordered.push_back(descs[k]);
  CUDA_TRY(cudaMemcpyAsync(d_descs, ordered.data(), sizeof(NetDesc) * n, cudaMemcpyHostToDevice, h0->stream));
  cudaError_t e = cudaSuccess;
  std::vector<cudaStream_t> forks;
  cudaEvent_t ready = nullptr;
  if (groups.size() > 1) {
    e = cudaEventCreateWithFlags(&ready, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(ready, h0->stream);
  }
  size_t off = 0;
  for (size_t gi = 0; gi < groups.size() && e == cudaSuccess; ++gi) {
    const std::vector<int>& g = groups[gi];
    snn::LaunchParams lp;
    std::memset(&lp, 0, sizeof(lp));
    lp.descs = d_descs + off;
    size_t smem = 0;
    bool lean = ev;
    for (int k : g) lean = lean && hs[k]->lean && hs[k]->p.wta_mode == hs[g[0]]->p.wta_mode;   // one WTA instance
    for (int k : g) smem = std::max(smem, lean ? hs[k]->smem_lean : hs[k]->smem);
    cudaStream_t st = h0->stream;
    if (groups.size() > 1) {
      e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
      if (e != cudaSuccess) break;
      forks.push_back(st);
      e = cudaStreamWaitEvent(st, ready, 0);
      if (e != cudaSuccess) break;
    }
    for (int k : g)
      if (hs[k]->nthr != hs[g[0]]->nthr) { e = cudaErrorInvalidValue; break; }
    if (e != cudaSuccess) break;
    for (int k : g)
      if (hs[k]->cpt != hs[g[0]]->cpt) { e = cudaErrorInvalidValue; break; }
    if (e != cudaSuccess) break;
    e = lean ? snn::launch_present_lean(lp, (int)g.size(), h0->cs, hs[g[0]]->nthr, smem, hs[g[0]]->bits,
                                        hs[g[0]]->cpt, h0->p.membrane_mode, hs[g[0]]->world > 1,
                                        hs[g[0]]->p.wta_mode == SNN_WTA_LAYER, st)
        : ev ? snn::launch_present_event_mode(lp, (int)g.size(), h0->cs, hs[g[0]]->nthr, smem, hs[g[0]]->bits,
                                              hs[g[0]]->cpt, h0->p.membrane_mode, st)
             : snn::launch_present(lp, (int)g.size(), h0->cs, h0->nthr, smem, st);
    off += g.size();
  }
  for (cudaStream_t st : forks) {
    cudaError_t e2 = cudaStreamSynchronize(st);
    if (e == cudaSuccess) e = e2;
    cudaStreamDestroy(st);
  }
  if (ready) cudaEventDestroy(ready);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h0->stream);
  cudaFree(d_descs);
  if (e != cudaSuccess) return fail(SNN_ECUDA, "present_many: %s", cudaGetErrorString(e));
  for (int k = 0; k < n; ++k) {
    hs[k]->launches++;
    if (infer) continue;
    hs[k]->last_T = T;
    hs[k]->last_recorded = false;
    hs[k]->t_next = T;
  }
  return SNN_OK;
}
}  // namespace

extern "C" {

int snn_present_many(snn_handle* const* hs, int n, const uint8_t* const* images, int n_images, int T,
                     const uint64_t* const* seeds) {
  return present_many_impl(hs, n, images, n_images, T, seeds, 0, nullptr);
}

int snn_infer_many(snn_handle* const* hs, int n, const uint8_t* const* images, int n_images, int T,
                   const uint64_t* const* seeds, uint32_t* const* counts) {
  if (!hs || n < 1 || !counts) return fail(SNN_EINVAL, "bad arguments");
  if (n_images < 0 || T < 0 || T > 65535) return fail(SNN_EINVAL, "n_images / T out of range");
  if (n_images == 0) return SNN_OK;
  std::vector<uint32_t*> dev(n, nullptr);
  for (int k = 0; k < n; ++k) {
    if (!hs[k] || !counts[k]) return fail(SNN_EINVAL, "handle / counts %d is NULL", k);
    if (is_device_ptr(counts[k])) { dev[k] = counts[k]; continue; }
    int rc = ensure(hs[k], &hs[k]->d_icounts, &hs[k]->icounts_cap, (size_t)n_images * hs[k]->n_exc);
    if (rc) return rc;
    dev[k] = hs[k]->d_icounts;
  }
  int rc = present_many_impl(hs, n, images, n_images, T, seeds, snn::FLAG_NO_LEARN, dev.data());
  if (rc) return rc;
  DevGuard g(hs[0]->dev);
  for (int k = 0; k < n; ++k) {      // inference counters (snn_get_infer_stats [0], [1]) and the host copies
    snn_handle* h = hs[k];
    if (!h->d_istats) {
      CUDA_TRY(dalloc(&h->d_istats, 3));
      CUDA_TRY(cudaMemset(h->d_istats, 0, 3 * sizeof(unsigned long long)));
    }
    unsigned long long sc[SNN_NSTATS], is[3];
    CUDA_TRY(cudaMemcpy(sc, h->d_iscratch, sizeof(sc), cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(is, h->d_istats, sizeof(is), cudaMemcpyDeviceToHost));
    is[0] += sc[0];
    is[1] += sc[1];
    CUDA_TRY(cudaMemcpy(h->d_istats, is, sizeof(is), cudaMemcpyHostToDevice));
    if (dev[k] != counts[k])
      CUDA_TRY(cudaMemcpy(counts[k], dev[k], (size_t)n_images * h->n_exc * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  }
  return SNN_OK;
}

int snn_get_weights(snn_handle* h, uint8_t* codes, size_t cap) {
  int rc = check_handle(h);
  if (rc) return rc;
  const size_t n = (size_t)h->n_in * h->n_exc * code_bytes(h->bits);     // bytes
  if (!codes) return fail(SNN_EINVAL, "codes is NULL");
  if (cap < n) return fail(SNN_ESIZE, "need %zu bytes", n);
  DevGuard g(h->dev);
  NetDesc d;
  fill_static(h, d);
  CUDA_TRY(snn::launch_unpack_weights(d, h->d_codes, h->stream));
  CUDA_TRY(cudaMemcpyAsync(codes, h->d_codes, n, is_device_ptr(codes) ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                           h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_set_weights(snn_handle* h, const uint8_t* codes, size_t n) {
  int rc = check_handle(h);
  if (rc) return rc;
  const size_t ncodes = (size_t)h->n_in * h->n_exc;
  const size_t need = ncodes * code_bytes(h->bits);                          // bytes
  if (!codes) return fail(SNN_EINVAL, "codes is NULL");
  if (n < need) return fail(SNN_ESIZE, "need %zu bytes", need);
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(h->d_codes, codes, need, is_device_ptr(codes) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                           h->stream));
  CUDA_TRY(cudaMemsetAsync(h->d_bad, 0, sizeof(int), h->stream));
  if (h->bits == 32)
    CUDA_TRY(snn::launch_check_g(reinterpret_cast<const float*>(h->d_codes), ncodes, (float)h->p.g_min, (float)h->p.g_max,
                                 h->d_bad, h->stream));
  else
    CUDA_TRY(snn::launch_check_codes(h->d_codes, ncodes, h->bits, h->q_max, h->d_bad, h->stream));
  int bad = 0;
  CUDA_TRY(cudaMemcpyAsync(&bad, h->d_bad, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  if (bad && h->bits == 32) return fail(SNN_EINVAL, "%d conductances outside [g_min, g_max] (R28)", bad);
  if (bad) return fail(SNN_EINVAL, "%d codes exceed q_max=%d", bad, h->q_max);
  NetDesc d;
  fill_static(h, d);
  CUDA_TRY(snn::launch_pack_weights(d, h->d_codes, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  h->w_version++;
  return SNN_OK;
}

int snn_get_spikes(snn_handle* h, uint32_t* raster, size_t cap_words) {
  int rc = check_handle(h);
  if (rc) return rc;
  const size_t need = (size_t)h->last_T * ((h->n_exc + 31) / 32);
  if (cap_words < need) return fail(SNN_ESIZE, "need %zu words", need);
  if (!need) return SNN_OK;
  if (!raster) return fail(SNN_EINVAL, "raster is NULL");
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(raster, h->d_raster, need * 4, cudaMemcpyDefault, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_get_input_raster(snn_handle* h, uint32_t* raster, size_t cap_words) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!h->last_recorded) return fail(SNN_EINVAL, "last presentation did not set SNN_RECORD_INPUT");
  const size_t need = (size_t)h->last_T * ((h->n_in + 31) / 32);
  if (cap_words < need) return fail(SNN_ESIZE, "need %zu words", need);
  if (!need) return SNN_OK;
  if (!raster) return fail(SNN_EINVAL, "raster is NULL");
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(raster, h->d_inrec, need * 4, cudaMemcpyDefault, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

size_t snn_state_bytes(const snn_handle* h) {
  if (!h) return 0;
  return sizeof(int32_t) * (4 + 3 * (size_t)h->n_exc + (size_t)h->n_in);
}

int snn_get_state(snn_handle* h, void* buf, size_t cap) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!buf) return fail(SNN_EINVAL, "buf is NULL");
  if (cap < snn_state_bytes(h)) return fail(SNN_ESIZE, "need %zu bytes", snn_state_bytes(h));
  DevGuard g(h->dev);
  int32_t* w = static_cast<int32_t*>(buf);
  const size_t ne = (size_t)h->n_exc;
  CUDA_TRY(cudaMemcpyAsync(w + 4, h->d_v, ne * 4, cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaMemcpyAsync(w + 4 + ne, h->d_cnt, ne * 4, cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaMemcpyAsync(w + 4 + 2 * ne, h->d_lpost, ne * 4, cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaMemcpyAsync(w + 4 + 3 * ne, h->d_lpre, (size_t)h->n_in * 4, cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  w[0] = h->n_in; w[1] = h->n_exc; w[2] = h->t_next; w[3] = h->p.membrane_mode;
  return SNN_OK;
}

int snn_set_state(snn_handle* h, const void* buf, size_t n) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!buf) return fail(SNN_EINVAL, "buf is NULL");
  if (n < snn_state_bytes(h)) return fail(SNN_ESIZE, "need %zu bytes", snn_state_bytes(h));
  const int32_t* w = static_cast<const int32_t*>(buf);
  if (w[0] != h->n_in || w[1] != h->n_exc || w[3] != h->p.membrane_mode || w[2] < 0)
    return fail(SNN_EINVAL, "state header does not match this handle");
  for (int j = 0; j < h->n_exc; ++j) {           // countdowns >= 0, spike timers NEVER or before t_next
    const int32_t c = w[4 + h->n_exc + j], lp = w[4 + 2 * h->n_exc + j];
    if (c < 0 || lp < snn::kNever || lp >= w[2]) return fail(SNN_EINVAL, "state: column %d has cnt %d / last_post %d", j, c, lp);
  }
  for (int i = 0; i < h->n_in; ++i) {
    const int32_t lp = w[4 + 3 * h->n_exc + i];
    if (lp < snn::kNever || lp >= w[2]) return fail(SNN_EINVAL, "state: input %d has last_pre %d (t_next %d)", i, lp, w[2]);
  }
  DevGuard g(h->dev);
  const size_t ne = (size_t)h->n_exc;
  CUDA_TRY(cudaMemcpyAsync(h->d_v, w + 4, ne * 4, cudaMemcpyHostToDevice, h->stream));
  CUDA_TRY(cudaMemcpyAsync(h->d_cnt, w + 4 + ne, ne * 4, cudaMemcpyHostToDevice, h->stream));
  CUDA_TRY(cudaMemcpyAsync(h->d_lpost, w + 4 + 2 * ne, ne * 4, cudaMemcpyHostToDevice, h->stream));
  CUDA_TRY(cudaMemcpyAsync(h->d_lpre, w + 4 + 3 * ne, (size_t)h->n_in * 4, cudaMemcpyHostToDevice, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  h->t_next = w[2];
  return SNN_OK;
}

int snn_get_stats(snn_handle* h, uint64_t stats[SNN_NSTATS]) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!stats) return fail(SNN_EINVAL, "stats is NULL");
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(stats, h->d_stats, SNN_NSTATS * sizeof(uint64_t), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_set_profile(snn_handle* h, int on) {
  int rc = check_handle(h);
  if (rc) return rc;
  h->prof = on != 0;
  h->prof_used = 0;
  return SNN_OK;
}

int snn_get_profile(snn_handle* h, double* kernel_ms, int64_t* kernels) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!kernel_ms || !kernels) return fail(SNN_EINVAL, "kernel_ms / kernels is NULL");
  DevGuard g(h->dev);
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  double ms = 0.0;
  for (size_t k = 0; k + 1 < h->prof_used; k += 2) {
    float x = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&x, h->prof_ev[k], h->prof_ev[k + 1]));
    ms += x;
  }
  *kernel_ms = ms;
  *kernels = (int64_t)(h->prof_used / 2);
  h->prof_used = 0;
  return SNN_OK;
}

int snn_reset_stats(snn_handle* h) {
  int rc = check_handle(h);
  if (rc) return rc;
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemsetAsync(h->d_stats, 0, SNN_NSTATS * sizeof(unsigned long long), h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_set_trace(snn_handle* h, int max_epochs) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (max_epochs < 0) return fail(SNN_EINVAL, "max_epochs < 0");
  DevGuard g(h->dev);
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  if (h->d_trace) cudaFree(h->d_trace);
  h->d_trace = nullptr;
  h->trace_epochs = 0;
  if (max_epochs > 0) {
    const size_t n = (size_t)h->cs * max_epochs * 8;
    CUDA_TRY(dalloc(&h->d_trace, n));
    CUDA_TRY(cudaMemset(h->d_trace, 0, n * sizeof(unsigned long long)));
    h->trace_epochs = max_epochs;
  }
  return SNN_OK;
}

int snn_get_trace(snn_handle* h, uint64_t* out, size_t cap) {
  int rc = check_handle(h);
  if (rc) return rc;
  const size_t n = (size_t)h->cs * h->trace_epochs * 8;
  if (!h->d_trace) return fail(SNN_EINVAL, "tracing is off (snn_set_trace)");
  if (!out || cap < n) return fail(SNN_ESIZE, "need %zu values", n);
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(out, h->d_trace, n * sizeof(uint64_t), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_get_info(const snn_handle* h, int64_t info[SNN_NINFO]) {
  if (!h || !info) return fail(SNN_EINVAL, "NULL argument");
  info[0] = h->cs; info[1] = h->nthr; info[2] = (int64_t)h->smem; info[3] = h->wpr;
  info[4] = h->q_max; info[5] = h->L_pot; info[6] = h->L_dep; info[7] = h->launches;
  info[8] = h->engine; info[9] = h->cpt; info[10] = h->rows_cap; info[11] = h->logn;
  info[12] = h->col_base; info[13] = h->n_exc_total; info[14] = h->world; info[15] = h->shard;
  info[16] = h->lean ? 1 : 0; info[17] = (int64_t)h->smem_lean;
  return SNN_OK;
}

}  // extern "C"

// ---------------------------------------------------------------- NEXT-1: inference, labelling, vote
namespace {

// Ring geometry of the inference kernel for this handle: the largest ring (multiple of 8, <= 64 rows;
// >= 32 rows) that leaves room for three CTAs per SM, else two, else one (>= 8 rows).  r01 sweep on
// 784->6400 2-bit (decoupled producer): R=40 / 3 CTAs 468k images/s, R=32 / 3 CTAs 448-455k, R=64 / 2 CTAs 401k,
// R=16 / 3 CTAs 133k (steps beyond R/2 rows take the direct path).
int infer_geometry(const snn_handle* h, int* wpr, int* R, int* nthr, size_t* smem) {
  const int ncols = (h->n_exc + 31) / 32;
  *wpr = ((ncols * h->bits) + 3) & ~3;
  const int row_bytes = *wpr * 4;
  *nthr = (((ncols + 31) / 32) + 1) * 32;
  int r = 64;
  if (const char* e = std::getenv("SNN_INFER_RING"))   // experiment hook: ring rows (multiple of 8, 8..64)
    if (std::atoi(e) >= 8 && std::atoi(e) <= 64 && !(std::atoi(e) & 7)) r = std::atoi(e);
  while (r > 32 && snn::infer_smem_bytes(r, row_bytes) > 74 * 1024) r -= 8;    // three CTAs per SM (measured best)
  while (r > 8 && snn::infer_smem_bytes(r, row_bytes) > 110 * 1024) r -= 8;
  while (r > 8 && snn::infer_smem_bytes(r, row_bytes) > 220 * 1024) r -= 8;
  if (snn::infer_smem_bytes(r, row_bytes) > 220 * 1024) return fail(SNN_ESIZE, "inference ring does not fit");
  *R = r;
  *smem = snn::infer_smem_bytes(r, row_bytes);
  return SNN_OK;
}

int infer_weights(snn_handle* h, int wpr) {
  if (h->infer_version == h->w_version && h->d_winf) return SNN_OK;
  int rc = ensure(h, &h->d_winf, &h->winf_cap, (size_t)h->n_in * wpr);
  if (rc) return rc;
  NetDesc d;
  fill_static(h, d);
  CUDA_TRY(snn::launch_unpack_weights(d, h->d_codes, h->stream));
  CUDA_TRY(snn::launch_pack_infer(h->d_codes, h->n_in, h->n_exc, h->bits, wpr, h->d_winf, h->stream));
  h->launches += 2;
  h->infer_version = h->w_version;
  return SNN_OK;
}

}  // namespace

extern "C" {

}  // extern "C"

namespace {
// Inference at 16 bits (R27) and with binary32 conductances (R28): the per-step engine's presentation kernel with
// FLAG_NO_LEARN (steps 1-4 of DESIGN.md §3.5 only, R21), images one after another on the handle's cluster, state
// reset per image (R5), spikes per neuron and image written by the kernel; the handle's weights and state are not
// touched.  Inference stats: [0] active input rows, [1] post spikes ([2], the LIF column-steps, is counted by the
// batch-parallel kernel of the <= 8-bit codes only).
int infer_step_engine(snn_handle* h, const uint8_t* images, int n_images, int T, const uint64_t* seeds,
                      uint32_t* counts, int flags) {
  if (n_images == 0) return SNN_OK;
  if (!images || !seeds || !counts) return fail(SNN_EINVAL, "images / seeds / counts is NULL");
  int rc;
  DevGuard g(h->dev);
  if (!h->d_istats) {
    CUDA_TRY(dalloc(&h->d_istats, 3));
    CUDA_TRY(cudaMemsetAsync(h->d_istats, 0, 3 * sizeof(unsigned long long), h->stream));
  }
  if (!h->d_iscratch) CUDA_TRY(dalloc(&h->d_iscratch, SNN_NSTATS));
  CUDA_TRY(cudaMemsetAsync(h->d_iscratch, 0, SNN_NSTATS * sizeof(unsigned long long), h->stream));
  const uint8_t* img = nullptr;
  if ((rc = stage(h, images, (size_t)n_images * h->n_in, &h->d_img, &h->img_cap, &img))) return rc;
  const unsigned long long* sd = nullptr;
  if ((rc = stage(h, reinterpret_cast<const unsigned long long*>(seeds), (size_t)n_images, &h->d_seeds,
                  &h->seeds_cap, &sd)))
    return rc;
  const bool counts_dev = is_device_ptr(counts);
  uint32_t* cnt = counts;
  if (!counts_dev) {
    if ((rc = ensure(h, &h->d_icounts, &h->icounts_cap, (size_t)n_images * h->n_exc))) return rc;
    cnt = h->d_icounts;
  }
  NetDesc d;
  fill_static(h, d);
  d.n_images = n_images; d.T = T; d.flags = snn::FLAG_NO_LEARN; d.t0 = 0;
  d.images = img; d.seeds = sd; d.neuron_counts = cnt; d.stats = h->d_iscratch;
  snn::LaunchParams lp;
  lp.descs = nullptr;
  lp.single = d;
  CUDA_TRY(snn::launch_present(lp, 1, h->cs, h->nthr, h->smem, h->stream));
  h->launches++;
  unsigned long long sc[SNN_NSTATS], is[3];
  CUDA_TRY(cudaMemcpyAsync(sc, h->d_iscratch, sizeof(sc), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaMemcpyAsync(is, h->d_istats, sizeof(is), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  is[0] += sc[0];
  is[1] += sc[1];
  CUDA_TRY(cudaMemcpyAsync(h->d_istats, is, sizeof(is), cudaMemcpyHostToDevice, h->stream));
  if (!counts_dev)
    CUDA_TRY(cudaMemcpyAsync(counts, cnt, (size_t)n_images * h->n_exc * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                             h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return finish(h, flags & ~SNN_ASYNC);
}
}  // namespace

extern "C" {

int snn_infer(snn_handle* h, const uint8_t* images, int n_images, int T, const uint64_t* seeds, uint32_t* counts,
              int flags) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (n_images < 0 || T < 0) return fail(SNN_EINVAL, "negative n_images / T");
  if (T > 65535) return fail(SNN_EINVAL, "T=%d exceeds 65535 for inference", T);
  if (h->world > 1) return fail(SNN_EINVAL, "inference runs on unsharded handles");
  if (h->bits > 8) return infer_step_engine(h, images, n_images, T, seeds, counts, flags);
  if (h->n_exc > snn::kInferMaxCols) return fail(SNN_ESIZE, "n_exc=%d exceeds %d for inference", h->n_exc,
                                                 snn::kInferMaxCols);
  if (n_images == 0) return SNN_OK;
  if (!images || !seeds || !counts) return fail(SNN_EINVAL, "images / seeds / counts is NULL");
  DevGuard g(h->dev);
  int wpr, R, nthr;
  size_t smem;
  if ((rc = infer_geometry(h, &wpr, &R, &nthr, &smem))) return rc;
  if ((rc = infer_weights(h, wpr))) return rc;
  if (!h->d_istats) {
    CUDA_TRY(dalloc(&h->d_istats, 3));
    CUDA_TRY(cudaMemsetAsync(h->d_istats, 0, 3 * sizeof(unsigned long long), h->stream));
  }
  const uint8_t* img = nullptr;
  if ((rc = stage(h, images, (size_t)n_images * h->n_in, &h->d_img, &h->img_cap, &img))) return rc;
  const unsigned long long* sd = nullptr;
  if ((rc = stage(h, reinterpret_cast<const unsigned long long*>(seeds), (size_t)n_images, &h->d_seeds,
                  &h->seeds_cap, &sd)))
    return rc;
  const bool counts_dev = is_device_ptr(counts);
  uint32_t* cnt = counts;
  if (!counts_dev) {
    if ((rc = ensure(h, &h->d_icounts, &h->icounts_cap, (size_t)n_images * h->n_exc))) return rc;
    cnt = h->d_icounts;
  }
  int minb = smem <= 74 * 1024 ? 3 : 2;           // register budget (<= 80 / <= 128) matching the smem occupancy
  if (const char* e = std::getenv("SNN_INFER_MINB"))   // experiment hook
    if (std::atoi(e) == 2 || std::atoi(e) == 3) minb = std::atoi(e);
  int occ = 0;
  CUDA_TRY(snn::infer_occupancy(h->bits, h->p.membrane_mode, minb, nthr, smem, &occ));
  if (occ < 1) return fail(SNN_ESIZE, "inference kernel cannot be resident (smem %zu B, %d threads)", smem, nthr);
  int nsm = 0;
  CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, h->dev));
  const int nwi = (h->n_in + 31) / 32;
  // the encoder pre-pass writes T x nwi words per image: process the batch in chunks of bounded scratch
  const long long per_img = (long long)T * nwi;
  const int chunk = (int)std::max(1LL, std::min<long long>(n_images, (256LL << 20) / 4 / std::max(1LL, per_img)));
  if ((rc = ensure(h, &h->d_iwords, &h->iwords_cap, (size_t)chunk * per_img))) return rc;
  if ((rc = ensure(h, &h->d_iecnt, &h->iecnt_cap, (size_t)chunk * T))) return rc;
  CUDA_TRY(cudaMemsetAsync(cnt, 0, (size_t)n_images * h->n_exc * sizeof(uint32_t), h->stream));
  snn::InferDesc d{};
  const snn_params& p = h->p;
  const double lsb = std::ldexp(1.0, -h->frac_bits);
  d.n_in = h->n_in; d.n_exc = h->n_exc; d.bits = h->bits; d.T = T; d.nwi = nwi;
  d.nthr_cols = (h->n_exc + 31) / 32; d.wpr = wpr; d.R = R; d.rmax = R / 2; d.row_bytes = wpr * 4;
  d.af = (float)p.a; d.bf = (float)p.b; d.cf = (float)p.c; d.dtf = (float)p.dt_ms;
  d.kI = (float)(p.v_spike * lsb); d.ief = (float)p.i_ext;
  d.vthf = (float)p.v_th; d.vresetf = (float)p.v_reset; d.vinitf = (float)p.v_init;
  d.A = h->A; d.B = h->B; d.C = h->C; d.E = h->E; d.Vth = h->Vth; d.Vreset = h->Vreset; d.Vinit = h->Vinit;
  d.t_ref = p.t_ref_steps; d.t_inh = p.t_inh_steps; d.wta_mode = p.wta_mode; d.inh_mode = p.inh_mode;
  d.w = h->d_winf; d.words = h->d_iwords; d.stats = h->d_istats;
  for (int k0 = 0; k0 < n_images; k0 += chunk) {
    const int nb = std::min(chunk, n_images - k0);
    CUDA_TRY(snn::launch_encode(img + (size_t)k0 * h->n_in, h->d_enc, sd + k0, h->n_in, T, nb, 0, h->d_iwords,
                                h->d_iecnt, h->stream));
    d.n_images = nb;
    d.counts = cnt + (size_t)k0 * h->n_exc;
    int grid = std::min(nb, occ * nsm);
    if (const char* e = std::getenv("SNN_INFER_MAX_GRID"))   // test hook: force the persistent image loop
      if (std::atoi(e) > 0) grid = std::min(grid, std::atoi(e));
    CUDA_TRY(snn::launch_infer(d, grid, nthr, smem, h->p.membrane_mode, minb, h->stream));
    h->launches += 2;
  }
  if (!counts_dev)
    CUDA_TRY(cudaMemcpyAsync(counts, cnt, (size_t)n_images * h->n_exc * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                             h->stream));
  return finish(h, flags);
}

int snn_get_infer_stats(snn_handle* h, uint64_t stats[3]) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!stats) return fail(SNN_EINVAL, "stats is NULL");
  stats[0] = stats[1] = stats[2] = 0;
  if (!h->d_istats) return SNN_OK;
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(stats, h->d_istats, 3 * sizeof(uint64_t), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

int snn_label(snn_handle* h, const uint32_t* counts, int n_images, const int32_t* classes, int n_classes,
              int32_t* labels) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!counts || !classes || !labels || n_images < 0) return fail(SNN_EINVAL, "bad labelling arguments");
  if (n_classes < 1 || n_classes > snn::kMaxClasses) return fail(SNN_EINVAL, "n_classes outside [1, %d]", snn::kMaxClasses);
  DevGuard g(h->dev);
  std::vector<int32_t> hc;
  if (!is_device_ptr(classes)) {       // validated on the host: a bad class id must not index out of bounds
    for (int k = 0; k < n_images; ++k)
      if (classes[k] < 0 || classes[k] >= n_classes) return fail(SNN_EINVAL, "classes[%d]=%d outside [0, %d)", k,
                                                                  classes[k], n_classes);
  } else {
    hc.resize((size_t)n_images);
    CUDA_TRY(cudaMemcpyAsync(hc.data(), classes, hc.size() * 4, cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    for (int k = 0; k < n_images; ++k)
      if (hc[k] < 0 || hc[k] >= n_classes) return fail(SNN_EINVAL, "classes[%d]=%d outside [0, %d)", k, hc[k], n_classes);
  }
  const uint32_t* c = nullptr;
  if ((rc = stage(h, counts, (size_t)n_images * h->n_exc, &h->d_icounts, &h->icounts_cap, &c))) return rc;
  const int32_t* cl = nullptr;
  if ((rc = stage(h, classes, (size_t)n_images, &h->d_cls, &h->cls_cap, &cl))) return rc;
  const bool out_dev = is_device_ptr(labels);
  int32_t* out = labels;
  if (!out_dev) {
    if ((rc = ensure(h, &h->d_lab, &h->lab_cap, (size_t)h->n_exc))) return rc;
    out = h->d_lab;
  }
  CUDA_TRY(snn::launch_label(c, n_images, h->n_exc, cl, n_classes, out, h->stream));
  h->launches++;
  if (!out_dev) CUDA_TRY(cudaMemcpyAsync(labels, out, (size_t)h->n_exc * 4, cudaMemcpyDeviceToHost, h->stream));
  return finish(h, 0);
}

int snn_classify(snn_handle* h, const uint32_t* counts, int n_images, const int32_t* labels, int n_classes,
                 int32_t* pred) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!counts || !labels || !pred || n_images < 0) return fail(SNN_EINVAL, "bad classification arguments");
  if (n_classes < 1 || n_classes > snn::kMaxClasses) return fail(SNN_EINVAL, "n_classes outside [1, %d]", snn::kMaxClasses);
  DevGuard g(h->dev);
  std::vector<int32_t> hl((size_t)h->n_exc);
  if (is_device_ptr(labels)) {
    CUDA_TRY(cudaMemcpyAsync(hl.data(), labels, hl.size() * 4, cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
  } else {
    std::memcpy(hl.data(), labels, hl.size() * 4);
  }
  for (int j = 0; j < h->n_exc; ++j)
    if (hl[j] < -1 || hl[j] >= n_classes) return fail(SNN_EINVAL, "labels[%d]=%d outside [-1, %d)", j, hl[j], n_classes);
  if (n_images == 0) return SNN_OK;
  const uint32_t* c = nullptr;
  if ((rc = stage(h, counts, (size_t)n_images * h->n_exc, &h->d_icounts, &h->icounts_cap, &c))) return rc;
  const int32_t* lb = nullptr;
  if ((rc = stage(h, labels, (size_t)h->n_exc, &h->d_lab, &h->lab_cap, &lb))) return rc;
  const bool out_dev = is_device_ptr(pred);
  int32_t* out = pred;
  if (!out_dev) {
    if ((rc = ensure(h, &h->d_cls, &h->cls_cap, (size_t)n_images))) return rc;
    out = h->d_cls;
  }
  CUDA_TRY(snn::launch_classify(c, n_images, h->n_exc, lb, n_classes, out, h->stream));
  h->launches++;
  if (!out_dev) CUDA_TRY(cudaMemcpyAsync(pred, out, (size_t)n_images * 4, cudaMemcpyDeviceToHost, h->stream));
  return finish(h, 0);
}

}  // extern "C"

// ---------------------------------------------------------------- NEXT-4: Fig. 4 sparse workload
extern "C" {

int snn_sparse_run(snn_handle* h, int n_lif, const int32_t* src_off, const uint16_t* tgt, const uint8_t* q,
                   const uint8_t* images, int n_trials, int T, const uint64_t* seeds, uint32_t* counts,
                   uint32_t* raster, int flags) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (n_lif < 1 || n_lif > snn::kSparseMaxLif) return fail(SNN_EINVAL, "n_lif=%d outside [1, %d]", n_lif, snn::kSparseMaxLif);
  if (n_trials < 0 || T < 0 || T > (1 << 30)) return fail(SNN_EINVAL, "bad n_trials / T");
  if (!src_off) return fail(SNN_EINVAL, "src_off is NULL");
  if (n_trials == 0) return SNN_OK;
  if (!images || !seeds || !counts) return fail(SNN_EINVAL, "images / seeds / counts is NULL");
  DevGuard g(h->dev);
  const int n_in = h->n_in, n_src = n_in + n_lif;
  // the graph is validated on the host (copied back first if it lives on the device)
  std::vector<int32_t> off((size_t)n_src + 1);
  if (is_device_ptr(src_off)) {
    CUDA_TRY(cudaMemcpy(off.data(), src_off, off.size() * 4, cudaMemcpyDeviceToHost));
  } else {
    std::memcpy(off.data(), src_off, off.size() * 4);
  }
  if (off[0] != 0) return fail(SNN_EINVAL, "src_off[0] must be 0");
  for (int s = 0; s < n_src; ++s)
    if (off[s + 1] < off[s]) return fail(SNN_EINVAL, "src_off not non-decreasing at %d", s);
  const size_t n_syn = (size_t)off[n_src];
  if (n_syn > 0 && (!tgt || !q)) return fail(SNN_EINVAL, "tgt / q is NULL");
  std::vector<uint16_t> ht(n_syn);
  std::vector<uint8_t> hq(n_syn);
  if (n_syn) {
    CUDA_TRY(cudaMemcpy(ht.data(), tgt, n_syn * 2, is_device_ptr(tgt) ? cudaMemcpyDeviceToHost : cudaMemcpyHostToHost));
    CUDA_TRY(cudaMemcpy(hq.data(), q, n_syn, is_device_ptr(q) ? cudaMemcpyDeviceToHost : cudaMemcpyHostToHost));
  }
  for (size_t k = 0; k < n_syn; ++k) {
    if (ht[k] >= n_lif) return fail(SNN_EINVAL, "tgt[%zu]=%d >= n_lif", k, (int)ht[k]);
    if (hq[k] > h->q_max) return fail(SNN_EINVAL, "q[%zu]=%d > q_max=%d", k, (int)hq[k], h->q_max);
  }
  if ((rc = ensure(h, &h->d_soff, &h->soff_cap, off.size()))) return rc;
  if ((rc = ensure(h, &h->d_stgt, &h->stgt_cap, std::max<size_t>(n_syn, 1)))) return rc;
  if ((rc = ensure(h, &h->d_sq, &h->sq_cap, std::max<size_t>(n_syn, 1)))) return rc;
  CUDA_TRY(cudaMemcpyAsync(h->d_soff, off.data(), off.size() * 4, cudaMemcpyHostToDevice, h->stream));
  if (n_syn) {
    CUDA_TRY(cudaMemcpyAsync(h->d_stgt, ht.data(), n_syn * 2, cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(cudaMemcpyAsync(h->d_sq, hq.data(), n_syn, cudaMemcpyHostToDevice, h->stream));
  }
  const uint8_t* img = nullptr;
  if ((rc = stage(h, images, (size_t)n_trials * n_in, &h->d_img, &h->img_cap, &img))) return rc;
  const unsigned long long* sd = nullptr;
  if ((rc = stage(h, reinterpret_cast<const unsigned long long*>(seeds), (size_t)n_trials, &h->d_seeds,
                  &h->seeds_cap, &sd)))
    return rc;
  const size_t n_counts = (size_t)n_trials * n_lif;
  const size_t n_raster = (size_t)n_trials * T * ((n_lif + 31) / 32);
  const bool counts_dev = is_device_ptr(counts);
  const bool raster_dev = raster && is_device_ptr(raster);
  uint32_t* dc = counts;
  uint32_t* dr = raster;
  if (!counts_dev) { if ((rc = ensure(h, &h->d_scounts, &h->scounts_cap, n_counts))) return rc; dc = h->d_scounts; }
  if (raster && !raster_dev) { if ((rc = ensure(h, &h->d_sraster, &h->sraster_cap, n_raster))) return rc; dr = h->d_sraster; }
  CUDA_TRY(cudaMemsetAsync(dc, 0, n_counts * 4, h->stream));
  if (dr) CUDA_TRY(cudaMemsetAsync(dr, 0, n_raster * 4, h->stream));
  if (!h->d_sstats) {
    CUDA_TRY(dalloc(&h->d_sstats, 2));
    CUDA_TRY(cudaMemsetAsync(h->d_sstats, 0, 2 * sizeof(unsigned long long), h->stream));
  }
  snn::SparseDesc d{};
  const snn_params& p = h->p;
  const double lsb = std::ldexp(1.0, -h->frac_bits);
  d.n_in = n_in; d.n_lif = n_lif; d.T = T; d.n_trials = n_trials; d.t_ref = p.t_ref_steps;
  d.af = (float)p.a; d.bf = (float)p.b; d.cf = (float)p.c; d.dtf = (float)p.dt_ms;
  d.kI = (float)(p.v_spike * lsb); d.ief = (float)p.i_ext;
  d.vthf = (float)p.v_th; d.vresetf = (float)p.v_reset; d.vinitf = (float)p.v_init;
  d.A = h->A; d.B = h->B; d.C = h->C; d.E = h->E; d.Vth = h->Vth; d.Vreset = h->Vreset; d.Vinit = h->Vinit;
  d.src_off = h->d_soff; d.tgt = h->d_stgt; d.q = h->d_sq; d.thr_enc = h->d_enc;
  d.images = img; d.seeds = sd; d.counts = dc; d.raster = dr; d.stats = h->d_sstats;
  const size_t smem = snn::sparse_smem_bytes(n_in, n_lif);
  const int nthr = std::max(128, std::min(512, ((n_lif + 31) / 32) * 32));   // threads stride over neurons
  int occ = 0, nsm = 0;
  CUDA_TRY(snn::sparse_occupancy(h->p.membrane_mode, nthr, smem, &occ));
  if (occ < 1) return fail(SNN_ESIZE, "sparse kernel cannot be resident (smem %zu B)", smem);
  CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, h->dev));
  CUDA_TRY(snn::launch_sparse(d, std::min(n_trials, occ * nsm), nthr, smem, h->p.membrane_mode, h->stream));
  h->launches++;
  if (!counts_dev) CUDA_TRY(cudaMemcpyAsync(counts, dc, n_counts * 4, cudaMemcpyDeviceToHost, h->stream));
  if (raster && !raster_dev) CUDA_TRY(cudaMemcpyAsync(raster, dr, n_raster * 4, cudaMemcpyDeviceToHost, h->stream));
  return finish(h, (counts_dev && (!raster || raster_dev)) ? flags : 0);
}

int snn_get_sparse_stats(snn_handle* h, uint64_t stats[2]) {
  int rc = check_handle(h);
  if (rc) return rc;
  if (!stats) return fail(SNN_EINVAL, "stats is NULL");
  stats[0] = stats[1] = 0;
  if (!h->d_sstats) return SNN_OK;
  DevGuard g(h->dev);
  CUDA_TRY(cudaMemcpyAsync(stats, h->d_sstats, 2 * sizeof(uint64_t), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return SNN_OK;
}

}  // extern "C"
