/*
 * snn_oracle.h -- CPU ORACLE for the simulate-and-learn loop of
 *   She, Long & Mukhopadhyay, "Fast and Low-Precision Learning in GPU-Accelerated
 *   Spiking Neural Network", DATE 2019  (/root/reference/PAPER.md, cited as P:<line>).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table builder or constant with the CUDA path (paper_conf_date_shelm19_b200/);
 * the parameter struct below is a hand-written duplicate of the layout documented in
 * DESIGN.md §3, not an include of include/snn.h.
 *
 * Plain, slow, single-threaded, obviously-correct loops in the paper's order.
 * Every reading of a silent / garbled passage is DESIGN.md §2 (R1..R20).
 */
#ifndef SNN_ORACLE_H
#define SNN_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct oracle_params {
  /* LIF eq.(1)(2), constants P:90 §III-D */
  double a, b, c, v_th, v_reset, v_init, dt_ms, v_spike, i_ext;
  int32_t t_ref_steps, t_inh_steps, wta_mode, inh_mode;
  /* encoder P:88 §III-B, Table I */
  double f_min_hz, f_max_hz;
  /* STDP: stdp_mode 0 = stochastic eqs.(6)(7) with dG = 1 LSB,
   *       1 = deterministic eqs.(4)(5) + rounding eq.(8)            */
  int32_t stdp_mode, rounding, t_ltp_steps, membrane_mode;
  double gamma_pot, tau_pot, gamma_dep, tau_dep;
  double alpha_p, beta_p, alpha_d, beta_d, g_min, g_max;
  int32_t frac_bits, init_mode;
  uint64_t init_seed;
  int32_t cluster_size, reserved0;
} oracle_params;

typedef struct oracle_net oracle_net;

/* Philox4x32-10 (Salmon et al., SC'11) -- the oracle's own copy. */
void oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);

int oracle_create(int n_in, int n_exc, int bits, const oracle_params* p, oracle_net** out);
int oracle_destroy(oracle_net* net);

/* flags */
#define ORACLE_RASTER_INPUT 1  /* `input` is a T x ceil(n_in/32) u32 spike raster, encoder bypassed */
#define ORACLE_KEEP_STATE   2  /* do not reset v/cnt/timers (R5); step indices start at t0 */

#define ORACLE_NO_LEARN     8  /* frozen weights: steps 1-4 only, no STDP (inference; R21) */

/* One presentation: T steps of the per-step loop.  image: n_in bytes (ignored with RASTER_INPUT). */
int oracle_present(oracle_net* net, const uint8_t* image, int T, uint64_t seed);
int oracle_present_ex(oracle_net* net, const void* input, int T, uint64_t seed, int flags, int t0);

/* codes n_in*n_exc row-major [i][j]: uint8 per code for bits <= 8, uint16 per code for bits = 16,
 * binary32 conductance G per synapse for bits = 32 (R28; set: every G in [G_min, G_max]) */
int oracle_get_weights(const oracle_net* net, void* codes);
int oracle_set_weights(oracle_net* net, const void* codes);
/* last presentation's output raster, T x ceil(n_exc/32) u32, bit j%32 of word j/32 */
int oracle_get_spikes(const oracle_net* net, uint32_t* raster, size_t cap_words);
/* last presentation's input raster, T x ceil(n_in/32) u32 */
int oracle_get_input_raster(const oracle_net* net, uint32_t* raster, size_t cap_words);
/* state blob, layout DESIGN.md §3.4: int32 header[4] = {n_in, n_exc, t_next, membrane_mode},
 * then v[n_exc] (float bits or Q15.16 int32), cnt[n_exc], last_post[n_exc], last_pre[n_in] (int32) */
size_t oracle_state_bytes(const oracle_net* net);
int oracle_get_state(const oracle_net* net, void* buf, size_t cap);
int oracle_set_state(oracle_net* net, const void* buf, size_t n);
/* counters of the last presentation: [0] sum_t act(t), [1] post spikes, [2] LTD trials,
 * [3] LTD events, [4] LTP trials, [5] LTP events */
int oracle_get_stats(const oracle_net* net, uint64_t stats[8]);

/* ---- NEXT-1: labelling and inference with frozen weights (§III-B "the first 1000 images in the
 * test set are used to label all the neurons in the first layer. The rest of the test set ... are used
 * for inference"; readings DESIGN.md R21-R23).
 * oracle_infer: each image presented for T steps with ORACLE_NO_LEARN, state reset per image (R5);
 *   counts[k*n_exc + j] = number of spikes of neuron j during image k.  Weights are not changed.
 * oracle_label: labels[j] = argmax_c (sum_{k: classes[k]==c} counts[k][j]) / N_c over classes with
 *   N_c > 0 images, ties -> lowest c; -1 if neuron j never spiked (R22).  classes[k] in [0, n_classes).
 * oracle_classify: pred[k] = argmax_c (sum_{j: labels[j]==c} counts[k][j]) / M_c over classes with
 *   M_c > 0 labelled neurons, ties -> lowest c; -1 if no labelled neuron spiked (R23).
 * Ratios are compared exactly as integer cross products. */
int oracle_infer(oracle_net* net, const uint8_t* images, int n_images, int T, const uint64_t* seeds,
                 uint32_t* counts);
int oracle_label(const uint32_t* counts, int n_images, int n_exc, const int32_t* classes, int n_classes,
                 int32_t* labels);
int oracle_classify(const uint32_t* counts, int n_images, int n_exc, const int32_t* labels, int n_classes,
                    int32_t* pred);

/* ---- NEXT-4: the Fig. 4 workload (§IV-A "an SNN of 10^3 LIF neurons and 10^4 synapses", no
 * learning; readings DESIGN.md R24-R26).  Sources 0..n_in-1 are the rate-coded input pixels (encoder as
 * in oracle_present, R8/R13), sources n_in..n_in+n_lif-1 are the LIF neurons themselves (recurrent, one
 * step of synaptic delay).  Synapse k of source s (k in [src_off[s], src_off[s+1])) targets LIF neuron
 * tgt[k] with code q[k] (G = q * 2^-bits, R9).  Per step t: S_j = sum of q[k] over synapses whose source
 * is active (input spike at t, or neuron spike at t-1); LIF recipe (membrane_mode) with refractory
 * t_ref; v > v_th -> spike, v = v_reset.  No WTA, no inhibition, no STDP.  State reset per trial (R5).
 * counts[k*n_lif + j] = spikes of neuron j in trial k; raster (optional, n_trials x T x ceil(n_lif/32)).
 * Uses the net's parameter block only (a, b, c, v_*, dt, v_spike, i_ext, t_ref, f_min/f_max, membrane
 * mode, bits). */
int oracle_sparse_run(const oracle_net* net, int n_in, int n_lif, const int32_t* src_off, const uint16_t* tgt,
                      const uint8_t* q, const uint8_t* images, int n_trials, int T, const uint64_t* seeds,
                      uint32_t* counts, uint32_t* raster);

/* Exposed for the pin tests. */
int oracle_q_max(const oracle_net* net);
int oracle_lut(const oracle_net* net, int which /*0 enc,1 pot,2 dep,3 det_p_base,4 det_p_thr,5 det_d_base,6 det_d_thr*/,
               uint64_t* out, int cap);
/* One LIF update (eq.(1) Euler, R2/R12) of a non-refractory neuron with integer synaptic sum S. */
float   oracle_lif_step_fp32(const oracle_net* net, float v, int32_t S);
int32_t oracle_lif_step_fixed(const oracle_net* net, int32_t v, int32_t S);
/* 32-bit floating-point conductance ("32-bit floating-point"; R28):
 * LIF update on the binary32 sum Sg = sum_i G_i; e^y by the binary64 recipe of R28; eqs.(4)(5) at G
 * (depress = 0: dG_p, 1: dG_d) in binary64. */
float   oracle_lif_step_fp32g(const oracle_net* net, float v, float Sg);
double  oracle_exp_recipe(const oracle_net* net, double y);
double  oracle_dg(const oracle_net* net, int depress, float G);

#ifdef __cplusplus
}
#endif
#endif
