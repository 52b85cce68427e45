/*
 * snn_oracle.c -- CPU ORACLE (test infrastructure; see snn_oracle.h header comment).
 *
 * Plain single-threaded C in the paper's order and notation.  What it follows:
 *   eq.(1)  dv/dt = a + b v + c I                       P:83 §II-A   (constants P:90 §III-D)
 *   eq.(2)  v = v_reset if v > v_threshold              P:83 §II-A
 *   eq.(3)  I_a = sum_n g_{n,a} v_pre,n                  P:83 §II-A
 *   rate encoder "proportional to the pixel intensity"   P:88 §III-B
 *   WTA: inhibit "all other neurons ... for t_inh"       P:88 §III-B
 *   eqs.(4)(5) deterministic dG (Querlioz [4])           P:84 §II-B
 *   eqs.(6)(7) P_pot = g_pot e^{-dt/t_pot}, P_dep = g_dep e^{dt/t_dep}   P:85 §II-C
 *   "For 8-bit and lower precision learning, dG is set to 1/2^n"        P:89 §III-C
 *   eq.(8)  P_round_up = (dG - dG_truncated) * 2^n       P:89 §III-C
 *   "spike timers", "fast CUDA random number generator"  P:87 §III-A  (-> Philox, R13)
 *   Table I parameters
 * Readings of silent/garbled passages: DESIGN.md §2, R1..R20 (cited inline as [Rn]).
 *
 * Compile with -ffp-contract=off (no implicit FMA): every fp32 rounding below is explicit.
 */
#include "snn_oracle.h"
#include <math.h>
#include <stdlib.h>
#include <string.h>

#define E_INVAL (-1)
#define E_NOMEM (-2)
#define E_SIZE  (-5)
#define NEVER   (-1)
#define LUT_MAX 4096

#define TAG_ENC   1u
#define TAG_LTD   2u
#define TAG_LTP   3u
#define TAG_ROUND 4u
#define TAG_INIT  5u
#define TAG_ROUND_LTD 6u   /* 16-bit stochastic arm: rounding draw of an LTD step [R27] */

/* Cody-Waite split of ln 2 (hi part has 11 trailing zero bits, so k * LN2_HI is exact for |k| < 2^11) and
 * 1/ln 2, as binary64 literals, for the exp recipe of the 32-bit arm [R28] */
#define INV_LN2 0x1.71547652b82fep+0
#define LN2_HI  0x1.62e42feep-1
#define LN2_LO  0x1.a39ef35793c76p-33
#define EXP_DEG 13

struct oracle_net {
  int n_in, n_exc, bits, frac_bits, q_max;
  oracle_params p;
  uint16_t* q;                /* conductance codes q[i*n_exc + j]; G = q * 2^-frac_bits [R9] (bits <= 16) */
  float* g;                   /* 32-bit arm: conductance G[i*n_exc + j] itself, IEEE binary32 [R28] */
  double ecoef[EXP_DEG + 1];  /* 1/m!, m = 0..EXP_DEG, by c_m = c_{m-1} / m in binary64 [R28] */
  float kV;                   /* (float) v_spike: I = v_spike * sum G, 32-bit arm [R28] */
  float gminf, gmaxf;
  /* state [R5] */
  float*   v_f;               /* membrane, fp32 mode */
  int32_t* v_x;               /* membrane, Q15.16 fixed mode */
  int32_t* cnt;               /* refractory / inhibition countdown [R6][R7] */
  int32_t* last_pre;          /* spike timers P:87 */
  int32_t* last_post;
  int32_t  t_next;
  /* probability tables [R13]: event iff u32 < thr */
  uint64_t thr_enc[256];
  uint64_t thr_pot[LUT_MAX]; int L_pot;
  uint64_t thr_dep[LUT_MAX]; int L_dep;
  /* eqs.(4)(5) magnitudes in LSB per code q (base + rounding threshold), q = 0..q_max [R16][R17]: the
   * deterministic arm at every width, and the stochastic arm's step size at 16 bits [R27] */
  int64_t* det_p_base; uint64_t* det_p_thr;
  int64_t* det_d_base; uint64_t* det_d_thr;
  /* fixed-point constants [R12] */
  int64_t A, B, C, E; int32_t Vth, Vreset, Vinit;
  /* fp32 constants [R12] */
  float af, bf, cf, dtf, kI, ief, vthf, vresetf, vinitf;
  /* last presentation outputs */
  uint32_t* raster;  int raster_T;
  uint32_t* in_raster;
  uint64_t stats[8];
};

/* ---------------------------------------------------------------- Philox4x32-10 [R13] */
/* Salmon, Moraes, Dror, Shaw, "Parallel random numbers: as easy as 1, 2, 3", SC'11:
 * round: (c0,c1,c2,c3) -> (hi(M1*c2)^c1^k0, lo(M1*c2), hi(M0*c0)^c3^k1, lo(M0*c0)),
 * key bump (k0,k1) += (W0,W1) between rounds; 10 rounds. */
void oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  const uint32_t M0 = 0xD2511F53u, M1 = 0xCD9E8D57u, W0 = 0x9E3779B9u, W1 = 0xBB67AE85u;
  uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int r = 0; r < 10; ++r) {
    if (r > 0) { k0 += W0; k1 += W1; }
    uint64_t p0 = (uint64_t)M0 * (uint64_t)c0;
    uint64_t p1 = (uint64_t)M1 * (uint64_t)c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0, n1 = lo1, n2 = hi0 ^ c3 ^ k1, n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* One uniform u32 from the counter layout of DESIGN.md §2 R13: lane `lane` of block ctr. */
static uint32_t draw(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t tag, int lane) {
  uint32_t ctr[4] = {c0, c1, c2, tag};
  uint32_t key[2] = {(uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32)};
  uint32_t out[4];
  oracle_philox4x32_10(ctr, key, out);
  return out[lane];
}

/* ---------------------------------------------------------------- tables */
/* thr = floor(P * 2^32), so that P(u32 < thr) = thr / 2^32 exactly [R13]. */
static uint64_t prob_to_thr(double P) { return (uint64_t)floor(ldexp(P, 32)); }

/* eqs.(6)(7): P_pot(D) = gamma_pot e^{-D dt/tau_pot}, D = t_post - t_pre >= 0;
 * P_dep(D) = gamma_dep e^{(-D) dt/tau_dep}, Dt = t_post - t_pre = -D < 0.  [R10][R11]
 * Length L = first D whose threshold is 0 (no event possible from there on). */
static int build_exp_lut(double gamma, double tau, double dt, uint64_t* thr, int* L) {
  *L = 0;
  if (gamma == 0.0) return 0;
  for (int D = 0; D < LUT_MAX; ++D) {
    uint64_t v = prob_to_thr(gamma * exp(-((double)D * dt) / tau));
    if (v == 0) { *L = D; return 0; }
    thr[D] = v;
  }
  return E_INVAL;  /* horizon longer than LUT_MAX steps: rejected */
}

static int validate(int n_in, int n_exc, int bits, const oracle_params* p) {
  if (n_in < 1 || n_in > 8192 || n_exc < 1 || n_exc > (1 << 20)) return E_INVAL;
  if (bits != 2 && bits != 4 && bits != 8 && bits != 16 && bits != 32) return E_INVAL;
  /* 32-bit floating-point conductance [R28]: fp32 membranes (the fixed recipe needs an integer sum) and
   * IEEE round-to-nearest (the trunc / eq.(8) roundings are defined on a fixed-point grid, R17) */
  if (bits == 32 && (p->membrane_mode != 0 || p->rounding != 1)) return E_INVAL;
  if (!(p->dt_ms > 0.0)) return E_INVAL;
  if (!(p->f_min_hz >= 0.0 && p->f_max_hz >= p->f_min_hz)) return E_INVAL;
  if (p->f_max_hz * p->dt_ms * 1e-3 > 1.0) return E_INVAL;
  if (!(p->gamma_pot >= 0.0 && p->gamma_pot <= 1.0 && p->gamma_dep >= 0.0 && p->gamma_dep <= 1.0)) return E_INVAL;
  if (!(p->tau_pot > 0.0 && p->tau_dep > 0.0)) return E_INVAL;
  if (p->t_ref_steps < 0 || p->t_inh_steps < 0 || p->t_ltp_steps < 0) return E_INVAL;
  if (p->wta_mode < 0 || p->wta_mode > 1 || p->inh_mode < 0 || p->inh_mode > 1) return E_INVAL;
  if (p->stdp_mode < 0 || p->stdp_mode > 1 || p->rounding < 0 || p->rounding > 2) return E_INVAL;
  if (p->membrane_mode < 0 || p->membrane_mode > 1) return E_INVAL;
  if (p->g_min != 0.0 || !(p->g_max > 0.0)) return E_INVAL;
  if (p->frac_bits < 0 || p->frac_bits > 16) return E_INVAL;
  if (p->init_mode != 0) return E_INVAL;
  if (p->stdp_mode == 1 && !(p->beta_p >= 0.0 && p->beta_d >= 0.0 && p->alpha_p >= 0.0 && p->alpha_d >= 0.0)) return E_INVAL;
  return 0;
}

int oracle_create(int n_in, int n_exc, int bits, const oracle_params* p, oracle_net** out) {
  if (!p || !out) return E_INVAL;
  int rc = validate(n_in, n_exc, bits, p);
  if (rc) return rc;
  oracle_net* n = (oracle_net*)calloc(1, sizeof(oracle_net));
  if (!n) return E_NOMEM;
  n->n_in = n_in; n->n_exc = n_exc; n->bits = bits; n->p = *p;
  /* [R9] G = q * 2^-frac_bits, frac_bits = bits unless given (Q1.7 style) */
  n->frac_bits = p->frac_bits > 0 ? p->frac_bits : bits;
  n->q_max = bits == 32 ? 0 : (1 << bits) - 1;   /* no code grid at 32 bits [R28] */
  if (bits <= 16 && n->frac_bits != bits) {
    double cap = floor(ldexp(p->g_max, n->frac_bits));
    if (cap < n->q_max) n->q_max = (int)cap;
  }
  double lsb = ldexp(1.0, -n->frac_bits);

  /* encoder table, P:88 + [R8]: f(x) = f_min + (f_max - f_min) x / 255, p = f dt */
  for (int x = 0; x < 256; ++x)
    n->thr_enc[x] = prob_to_thr((p->f_min_hz + (p->f_max_hz - p->f_min_hz) * (double)x / 255.0) * p->dt_ms * 1e-3);
  if (build_exp_lut(p->gamma_pot, p->tau_pot, p->dt_ms, n->thr_pot, &n->L_pot) ||
      build_exp_lut(p->gamma_dep, p->tau_dep, p->dt_ms, n->thr_dep, &n->L_dep)) { free(n); return E_INVAL; }

  /* eqs.(4)(5) in units of LSB, rounded by eq.(8) / trunc / nearest [R16][R17] */
  n->det_p_base = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n->q_max + 1));
  n->det_d_base = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n->q_max + 1));
  n->det_p_thr = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(n->q_max + 1));
  n->det_d_thr = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(n->q_max + 1));
  if (!n->det_p_base || !n->det_d_base || !n->det_p_thr || !n->det_d_thr) { oracle_destroy(n); return E_NOMEM; }
  for (int qq = 0; qq <= n->q_max; ++qq) {
    double G = (double)qq * lsb;
    double xp = ldexp(p->alpha_p * exp(-p->beta_p * (G - p->g_min) / (p->g_max - p->g_min)), n->frac_bits);
    double xd = ldexp(p->alpha_d * exp(-p->beta_d * (p->g_max - G) / (p->g_max - p->g_min)), n->frac_bits);
    double xs[2] = {xp, xd};
    for (int s = 0; s < 2; ++s) {
      double x = xs[s];
      int64_t base; uint64_t thr;
      if (p->rounding == 0)      { base = (int64_t)floor(x);       thr = 0; }              /* truncation */
      else if (p->rounding == 1) { base = (int64_t)floor(x + 0.5); thr = 0; }              /* nearest, half up */
      else                       { base = (int64_t)floor(x); thr = prob_to_thr(x - floor(x)); } /* eq.(8) */
      if (s == 0) { n->det_p_base[qq] = base; n->det_p_thr[qq] = thr; }
      else        { n->det_d_base[qq] = base; n->det_d_thr[qq] = thr; }
    }
  }

  /* fixed-point recipe [R12]: v Q15.16; A,E Q.16; B,C Q.32 */
  n->A = llround(p->dt_ms * p->a * 65536.0);
  n->B = llround(p->dt_ms * p->b * 4294967296.0);
  n->C = llround(p->dt_ms * p->c * p->v_spike * lsb * 4294967296.0);
  n->E = llround(p->dt_ms * p->c * p->i_ext * 65536.0);
  n->Vth = (int32_t)llround(p->v_th * 65536.0);
  n->Vreset = (int32_t)llround(p->v_reset * 65536.0);
  n->Vinit = (int32_t)llround(p->v_init * 65536.0);
  /* fp32 recipe [R12] */
  n->af = (float)p->a; n->bf = (float)p->b; n->cf = (float)p->c; n->dtf = (float)p->dt_ms;
  n->kI = (float)(p->v_spike * lsb); n->ief = (float)p->i_ext;
  n->vthf = (float)p->v_th; n->vresetf = (float)p->v_reset; n->vinitf = (float)p->v_init;
  /* 32-bit arm [R28] */
  n->kV = (float)p->v_spike; n->gminf = (float)p->g_min; n->gmaxf = (float)p->g_max;
  n->ecoef[0] = 1.0;
  for (int m = 1; m <= EXP_DEG; ++m) n->ecoef[m] = n->ecoef[m - 1] / (double)m;

  size_t nq = (size_t)n_in * (size_t)n_exc;
  n->q = (uint16_t*)malloc(nq * sizeof(uint16_t));
  if (bits == 32) {
    n->g = (float*)malloc(nq * sizeof(float));
    if (!n->g) { oracle_destroy(n); return E_NOMEM; }
  }
  n->v_f = (float*)calloc((size_t)n_exc, sizeof(float));
  n->v_x = (int32_t*)calloc((size_t)n_exc, sizeof(int32_t));
  n->cnt = (int32_t*)calloc((size_t)n_exc, sizeof(int32_t));
  n->last_post = (int32_t*)calloc((size_t)n_exc, sizeof(int32_t));
  n->last_pre = (int32_t*)calloc((size_t)n_in, sizeof(int32_t));
  if (!n->q || !n->v_f || !n->v_x || !n->cnt || !n->last_post || !n->last_pre) { oracle_destroy(n); return E_NOMEM; }

  /* initial conductance [R4]: P:90 is truncated ("initialized with  "); uniform codes */
  for (int i = 0; i < n_in; ++i)
    for (int j = 0; j < n_exc; ++j) {
      uint32_t u = draw(p->init_seed, (uint32_t)i, (uint32_t)(j >> 2), 0u, TAG_INIT, j & 3);
      n->q[(size_t)i * n_exc + j] = (uint16_t)(((uint64_t)u * (uint64_t)(n->q_max + 1)) >> 32);
      /* 32-bit arm [R28]: G = g_max * (u >> 8) 2^-24, uniform on the 2^24-point grid of [0, g_max) */
      if (bits == 32) n->g[(size_t)i * n_exc + j] = (float)(p->g_max * ldexp((double)(u >> 8), -24));
    }
  /* state as after a reset [R5] */
  for (int j = 0; j < n_exc; ++j) { n->v_f[j] = n->vinitf; n->v_x[j] = n->Vinit; n->last_post[j] = NEVER; }
  for (int i = 0; i < n_in; ++i) n->last_pre[i] = NEVER;
  *out = n;
  return 0;
}

int oracle_destroy(oracle_net* n) {
  if (!n) return 0;
  free(n->q); free(n->g); free(n->v_f); free(n->v_x); free(n->cnt); free(n->last_post); free(n->last_pre);
  free(n->raster); free(n->in_raster);
  free(n->det_p_base); free(n->det_d_base); free(n->det_p_thr); free(n->det_d_thr);
  free(n);
  return 0;
}

/* ---------------------------------------------------------------- LIF, eq.(1) forward Euler [R1][R2][R12] */
float oracle_lif_step_fp32(const oracle_net* n, float v, int32_t S) {
  float I  = (float)S * n->kI;            /* eq.(3): I = v_spike * sum_i G_i, G_i = q_i * LSB [R3] */
  float x  = I + n->ief;
  float y  = fmaf(n->cf, x, n->af);       /* a + c I */
  float dv = fmaf(n->bf, v, y);           /* a + b v + c I */
  return fmaf(n->dtf, dv, v);             /* v + dt dv/dt */
}

/* 32-bit arm [R28]: the same recipe on the binary32 conductance sum Sg = sum_i G_i (eq.(3): I = v_spike Sg) */
float oracle_lif_step_fp32g(const oracle_net* n, float v, float Sg) {
  float I  = Sg * n->kV;
  float x  = I + n->ief;
  float y  = fmaf(n->cf, x, n->af);
  float dv = fmaf(n->bf, v, y);
  return fmaf(n->dtf, dv, v);
}

/* e^y in binary64 by an explicit recipe [R28] (so that both implementations round identically):
 * y = k ln2 + r with k = nearest integer to y / ln2 and r = (y - k LN2_HI) - k LN2_LO (two fused
 * multiply-adds), e^r by its Taylor series to degree EXP_DEG in Horner form (fused multiply-adds), times 2^k.
 * |r| <= ln2 / 2 bounds the truncation error by 0.35^14 / 14! < 1e-17 relative (tests pin it to libm exp). */
double oracle_exp_recipe(const oracle_net* n, double y) {
  double k = nearbyint(y * INV_LN2);
  double r = fma(-k, LN2_HI, y);
  r = fma(-k, LN2_LO, r);
  double e = n->ecoef[EXP_DEG];
  for (int m = EXP_DEG - 1; m >= 0; --m) e = fma(e, r, n->ecoef[m]);
  return ldexp(e, (int)k);
}

/* eqs.(4)(5) at conductance G (binary64) [R28]:
 *   dG_p = alpha_p e^{-beta_p (G - G_min) / (G_max - G_min)},  dG_d = alpha_d e^{-beta_d (G_max - G) / (G_max - G_min)} */
double oracle_dg(const oracle_net* n, int depress, float G) {
  const oracle_params* p = &n->p;
  const double span = p->g_max - p->g_min;
  if (!depress) return p->alpha_p * oracle_exp_recipe(n, -p->beta_p * ((double)G - p->g_min) / span);
  return p->alpha_d * oracle_exp_recipe(n, -p->beta_d * (p->g_max - (double)G) / span);
}

/* P:89 "after floating point calculation of change in conductance dG, the result is rounded to a value that
 * can be represented in the current bit width": G' = binary32(G +- dG) (round to nearest), clamped to
 * [G_min, G_max] [R28] */
static float g_step(const oracle_net* n, float G, double dG, int depress) {
  float G1 = (float)(depress ? (double)G - dG : (double)G + dG);
  if (G1 < n->gminf) G1 = n->gminf;
  if (G1 > n->gmaxf) G1 = n->gmaxf;
  return G1;
}

int32_t oracle_lif_step_fixed(const oracle_net* n, int32_t v, int32_t S) {
  int64_t bv = (n->B * (int64_t)v + ((int64_t)1 << 31)) >> 32;   /* dt b v      (Q.16) */
  int64_t cs = (n->C * (int64_t)S + ((int64_t)1 << 15)) >> 16;   /* dt c v_spike LSB S */
  return (int32_t)((int64_t)v + n->A + bv + cs + n->E);
}

static void reset_state(oracle_net* n) {
  for (int j = 0; j < n->n_exc; ++j) {
    n->v_f[j] = n->vinitf; n->v_x[j] = n->Vinit; n->cnt[j] = 0; n->last_post[j] = NEVER;
  }
  for (int i = 0; i < n->n_in; ++i) n->last_pre[i] = NEVER;
}

int oracle_present(oracle_net* n, const uint8_t* image, int T, uint64_t seed) {
  return oracle_present_ex(n, image, T, seed, 0, 0);
}

int oracle_present_ex(oracle_net* n, const void* input, int T, uint64_t seed, int flags, int t0) {
  if (!n || T < 0 || t0 < 0 || (T > 0 && !input)) return E_INVAL;
  /* continuing a presentation may not step back in time: every stored timer is below t_next <= t0, so
   * Dt = t - last >= 1 indexes the eqs.(6)(7) tables (input validation, not part of the method) */
  if ((flags & ORACLE_KEEP_STATE) && t0 < n->t_next) return E_INVAL;
  const oracle_params* p = &n->p;
  const int n_in = n->n_in, n_exc = n->n_exc;
  const int wi = (n_in + 31) / 32, we = (n_exc + 31) / 32;
  const int fixed = p->membrane_mode == 1;

  if (!(flags & ORACLE_KEEP_STATE)) reset_state(n);           /* [R5] */
  free(n->raster); free(n->in_raster);
  n->raster = (uint32_t*)calloc((size_t)(T > 0 ? T : 1) * we, sizeof(uint32_t));
  n->in_raster = (uint32_t*)calloc((size_t)(T > 0 ? T : 1) * wi, sizeof(uint32_t));
  n->raster_T = T;
  memset(n->stats, 0, sizeof(n->stats));

  uint8_t* s = (uint8_t*)calloc((size_t)n_in, 1);
  int32_t* S = (int32_t*)calloc((size_t)n_exc, sizeof(int32_t));
  float* Sg = (float*)calloc((size_t)n_exc, sizeof(float));
  uint8_t* cand = (uint8_t*)calloc((size_t)n_exc, 1);
  int* spikers = (int*)malloc(sizeof(int) * (size_t)n_exc);
  if (!n->raster || !n->in_raster || !s || !S || !Sg || !cand || !spikers) {
    free(s); free(S); free(Sg); free(cand); free(spikers); return E_NOMEM;
  }

  for (int k = 0; k < T; ++k) {
    const int t = t0 + k;

    /* 1 ENCODE -- P:88 "Pixel intensity ... encoded into specific spiking frequency" [R8][R13] */
    for (int i = 0; i < n_in; ++i) {
      if (flags & ORACLE_RASTER_INPUT) {
        const uint32_t* r = (const uint32_t*)input;
        s[i] = (uint8_t)((r[(size_t)k * wi + i / 32] >> (i % 32)) & 1u);
      } else {
        uint32_t u = draw(seed, (uint32_t)t, (uint32_t)(i >> 2), 0u, TAG_ENC, i & 3);
        s[i] = (uint8_t)((uint64_t)u < n->thr_enc[((const uint8_t*)input)[i]]);
      }
      if (s[i]) {
        n->last_pre[i] = t;                                          /* spike timer P:87 */
        n->in_raster[(size_t)k * wi + i / 32] |= 1u << (i % 32);
        n->stats[0]++;
      }
    }

    /* 2 INTEGRATE -- eq.(3): S_j = sum over spiking pre-neurons of q[i][j] (I = v_spike LSB S);
     * 32-bit arm: Sg_j = sum of G[i][j] in binary32, ascending i [R28] */
    for (int j = 0; j < n_exc; ++j) {
      int32_t acc = 0;
      float accg = 0.0f;
      for (int i = 0; i < n_in; ++i) {
        if (!s[i]) continue;
        if (n->bits == 32) accg = accg + n->g[(size_t)i * n_exc + j];
        else acc += n->q[(size_t)i * n_exc + j];
      }
      S[j] = acc;
      Sg[j] = accg;
    }

    /* 3 LIF -- eqs.(1)(2); refractory/inhibited neurons hold v [R6][R7] */
    for (int j = 0; j < n_exc; ++j) {
      if (n->cnt[j] > 0) { n->cnt[j]--; cand[j] = 0; continue; }
      if (fixed) { n->v_x[j] = oracle_lif_step_fixed(n, n->v_x[j], S[j]); cand[j] = n->v_x[j] > n->Vth; }
      else if (n->bits == 32) { n->v_f[j] = oracle_lif_step_fp32g(n, n->v_f[j], Sg[j]); cand[j] = n->v_f[j] > n->vthf; }
      else       { n->v_f[j] = oracle_lif_step_fp32(n, n->v_f[j], S[j]);  cand[j] = n->v_f[j] > n->vthf; }
    }

    /* 4 WTA -- P:88 layer-2 neuron inhibits "all other neurons on the first layer for t_inh" [R7] */
    int nsp = 0;
    if (p->wta_mode == 0) {            /* HARD: the largest margin v - v_th wins, ties -> lowest j */
      int W = -1;
      for (int j = 0; j < n_exc; ++j) {
        if (!cand[j]) continue;
        if (W < 0) { W = j; continue; }
        if (fixed ? (n->v_x[j] > n->v_x[W]) : (n->v_f[j] > n->v_f[W])) W = j;
      }
      if (W >= 0) spikers[nsp++] = W;
    } else {                           /* LAYER: every crossing neuron spikes */
      for (int j = 0; j < n_exc; ++j) if (cand[j]) spikers[nsp++] = j;
    }
    for (int m = 0; m < nsp; ++m) {
      int j = spikers[m];
      n->v_f[j] = n->vresetf; n->v_x[j] = n->Vreset;                 /* eq.(2) */
      n->cnt[j] = p->t_ref_steps;
      n->raster[(size_t)k * we + j / 32] |= 1u << (j % 32);
      n->stats[1]++;
    }
    if (nsp > 0) {
      for (int j = 0; j < n_exc; ++j) {
        int other = (nsp >= 2) || (j != spikers[0]);
        if (!other) continue;
        if (n->cnt[j] < p->t_inh_steps) n->cnt[j] = p->t_inh_steps;
        if (p->inh_mode == 0) { n->v_f[j] = n->vresetf; n->v_x[j] = n->Vreset; }
      }
    }

    /* 5 STDP (skipped with frozen weights: inference, R21) */
    if (flags & ORACLE_NO_LEARN) {
      /* no plasticity */
    } else if (p->stdp_mode == 0) {
      /* LTD at a pre spike against the last post spike, eq.(7), Dt = -D < 0 [R10][R14]; dG = 1 LSB */
      for (int i = 0; i < n_in; ++i) {
        if (!s[i]) continue;
        for (int j = 0; j < n_exc; ++j) {
          if (n->last_post[j] == NEVER) continue;
          int D = t - n->last_post[j];
          if (D >= n->L_dep) continue;
          n->stats[2]++;
          uint32_t u = draw(seed, (uint32_t)t, (uint32_t)i, (uint32_t)(j >> 2), TAG_LTD, j & 3);
          if ((uint64_t)u < n->thr_dep[D]) {
            n->stats[3]++;
            uint16_t* qq = &n->q[(size_t)i * n_exc + j];
            if (n->bits == 32) {                       /* 32 bit: G -= eq.(5), binary32 [R28] */
              float* g = &n->g[(size_t)i * n_exc + j];
              *g = g_step(n, *g, oracle_dg(n, 1, *g), 1);
            } else if (n->bits <= 8) {
              if (*qq > 0) *qq -= 1;                   /* dG = 1 LSB */
            } else {                                   /* 16 bit: dG = eq.(5), rounded (eq.(8)) [R27] */
              uint32_t u2 = draw(seed, (uint32_t)t, (uint32_t)i, (uint32_t)(j >> 2), TAG_ROUND_LTD, j & 3);
              int64_t dq = n->det_d_base[*qq] + ((uint64_t)u2 < n->det_d_thr[*qq] ? 1 : 0);
              int64_t q1 = (int64_t)*qq - dq;
              *qq = (uint16_t)(q1 < 0 ? 0 : q1);
            }
          }
        }
      }
      /* LTP at a post spike against the last pre spike, eq.(6), Dt = D >= 0 [R10][R14] */
      for (int m = 0; m < nsp; ++m) {
        int W = spikers[m];
        for (int i = 0; i < n_in; ++i) {
          if (n->last_pre[i] == NEVER) continue;
          int D = t - n->last_pre[i];
          if (D >= n->L_pot) continue;
          n->stats[4]++;
          uint32_t u = draw(seed, (uint32_t)t, (uint32_t)W, (uint32_t)(i >> 2), TAG_LTP, i & 3);
          if ((uint64_t)u < n->thr_pot[D]) {
            n->stats[5]++;
            uint16_t* qq = &n->q[(size_t)i * n_exc + W];
            if (n->bits == 32) {                       /* 32 bit: G += eq.(4), binary32 [R28] */
              float* g = &n->g[(size_t)i * n_exc + W];
              *g = g_step(n, *g, oracle_dg(n, 0, *g), 0);
            } else if (n->bits <= 8) {
              if (*qq < n->q_max) *qq += 1;            /* dG = 1 LSB */
            } else {                                   /* 16 bit: dG = eq.(4), rounded (eq.(8)) [R27] */
              uint32_t u2 = draw(seed, (uint32_t)t, (uint32_t)W, (uint32_t)(i >> 2), TAG_ROUND, i & 3);
              int64_t dq = n->det_p_base[*qq] + ((uint64_t)u2 < n->det_p_thr[*qq] ? 1 : 0);
              int64_t q1 = (int64_t)*qq + dq;
              *qq = (uint16_t)(q1 > n->q_max ? n->q_max : q1);
            }
          }
        }
      }
    } else {
      /* deterministic arm: at each post spike, eq.(4) inside the LTP window, eq.(5) outside,
       * magnitude rounded to the grid by trunc / nearest / eq.(8) [R16][R17] */
      for (int m = 0; m < nsp; ++m) {
        int W = spikers[m];
        for (int i = 0; i < n_in; ++i) {
          uint16_t* qq = &n->q[(size_t)i * n_exc + W];
          int q0 = *qq;
          int pot = n->last_pre[i] != NEVER && (t - n->last_pre[i]) <= p->t_ltp_steps;
          if (n->bits == 32) {                         /* eq.(4) or eq.(5) in binary32, no draw [R28] */
            float* g = &n->g[(size_t)i * n_exc + W];
            double dG = oracle_dg(n, !pot, *g);
            *g = g_step(n, *g, dG, !pot);
            n->stats[pot ? 4 : 2]++;
            if (dG > 0.0) n->stats[pot ? 5 : 3]++;
            continue;
          }
          int64_t base = pot ? n->det_p_base[q0] : n->det_d_base[q0];
          uint64_t thr = pot ? n->det_p_thr[q0] : n->det_d_thr[q0];
          uint32_t u = draw(seed, (uint32_t)t, (uint32_t)W, (uint32_t)(i >> 2), TAG_ROUND, i & 3);
          int64_t dq = base + ((uint64_t)u < thr ? 1 : 0);
          int64_t q1 = pot ? q0 + dq : q0 - dq;
          if (q1 < 0) q1 = 0;
          if (q1 > n->q_max) q1 = n->q_max;
          *qq = (uint16_t)q1;
          n->stats[pot ? 4 : 2]++;
          if (dq > 0) n->stats[pot ? 5 : 3]++;
        }
      }
    }
    for (int m = 0; m < nsp; ++m) n->last_post[spikers[m]] = t;      /* spike timer P:87 */
  }
  n->t_next = t0 + T;
  free(s); free(S); free(Sg); free(cand); free(spikers);
  return 0;
}

/* ---------------------------------------------------------------- accessors */
/* codes: one byte per code (bits <= 8), one uint16 per code (bits = 16), one binary32 G (bits = 32) */
int oracle_get_weights(const oracle_net* n, void* codes) {
  if (!n || !codes) return E_INVAL;
  size_t nq = (size_t)n->n_in * n->n_exc;
  if (n->bits == 32) { memcpy(codes, n->g, nq * sizeof(float)); return 0; }
  if (n->bits > 8) { memcpy(codes, n->q, nq * sizeof(uint16_t)); return 0; }
  for (size_t k = 0; k < nq; ++k) ((uint8_t*)codes)[k] = (uint8_t)n->q[k];
  return 0;
}

int oracle_set_weights(oracle_net* n, const void* codes) {
  if (!n || !codes) return E_INVAL;
  size_t nq = (size_t)n->n_in * n->n_exc;
  if (n->bits == 32) {                             /* every G finite and inside [G_min, G_max] [R28] */
    const float* g = (const float*)codes;
    for (size_t k = 0; k < nq; ++k) if (!(g[k] >= n->gminf && g[k] <= n->gmaxf)) return E_INVAL;
    memcpy(n->g, g, nq * sizeof(float));
    return 0;
  }
  for (size_t k = 0; k < nq; ++k) {
    int c = n->bits > 8 ? ((const uint16_t*)codes)[k] : ((const uint8_t*)codes)[k];
    if (c > n->q_max) return E_INVAL;
  }
  for (size_t k = 0; k < nq; ++k) n->q[k] = n->bits > 8 ? ((const uint16_t*)codes)[k] : ((const uint8_t*)codes)[k];
  return 0;
}

int oracle_get_spikes(const oracle_net* n, uint32_t* raster, size_t cap_words) {
  if (!n || (!raster && cap_words)) return E_INVAL;
  size_t need = (size_t)n->raster_T * ((n->n_exc + 31) / 32);
  if (cap_words < need) return E_SIZE;
  if (need) memcpy(raster, n->raster, need * sizeof(uint32_t));
  return 0;
}

int oracle_get_input_raster(const oracle_net* n, uint32_t* raster, size_t cap_words) {
  if (!n || (!raster && cap_words)) return E_INVAL;
  size_t need = (size_t)n->raster_T * ((n->n_in + 31) / 32);
  if (cap_words < need) return E_SIZE;
  if (need) memcpy(raster, n->in_raster, need * sizeof(uint32_t));
  return 0;
}

size_t oracle_state_bytes(const oracle_net* n) {
  return sizeof(int32_t) * (4 + 3 * (size_t)n->n_exc + (size_t)n->n_in);
}

int oracle_get_state(const oracle_net* n, void* buf, size_t cap) {
  if (!n || !buf) return E_INVAL;
  if (cap < oracle_state_bytes(n)) return E_SIZE;
  int32_t* w = (int32_t*)buf;
  w[0] = n->n_in; w[1] = n->n_exc; w[2] = n->t_next; w[3] = n->p.membrane_mode;
  int32_t* v = w + 4;
  for (int j = 0; j < n->n_exc; ++j) {
    if (n->p.membrane_mode == 1) v[j] = n->v_x[j];
    else memcpy(&v[j], &n->v_f[j], 4);
  }
  memcpy(w + 4 + n->n_exc, n->cnt, 4 * (size_t)n->n_exc);
  memcpy(w + 4 + 2 * (size_t)n->n_exc, n->last_post, 4 * (size_t)n->n_exc);
  memcpy(w + 4 + 3 * (size_t)n->n_exc, n->last_pre, 4 * (size_t)n->n_in);
  return 0;
}

int oracle_set_state(oracle_net* n, const void* buf, size_t sz) {
  if (!n || !buf) return E_INVAL;
  if (sz < oracle_state_bytes(n)) return E_SIZE;
  const int32_t* w = (const int32_t*)buf;
  if (w[0] != n->n_in || w[1] != n->n_exc || w[3] != n->p.membrane_mode || w[2] < 0) return E_INVAL;
  /* countdowns >= 0; spike timers NEVER or before t_next (input validation) */
  for (int j = 0; j < n->n_exc; ++j) {
    const int32_t c = w[4 + n->n_exc + j], lp = w[4 + 2 * n->n_exc + j];
    if (c < 0 || lp < NEVER || lp >= w[2]) return E_INVAL;
  }
  for (int i = 0; i < n->n_in; ++i) {
    const int32_t lp = w[4 + 3 * n->n_exc + i];
    if (lp < NEVER || lp >= w[2]) return E_INVAL;
  }
  n->t_next = w[2];
  const int32_t* v = w + 4;
  for (int j = 0; j < n->n_exc; ++j) {
    if (n->p.membrane_mode == 1) n->v_x[j] = v[j];
    else memcpy(&n->v_f[j], &v[j], 4);
  }
  memcpy(n->cnt, w + 4 + n->n_exc, 4 * (size_t)n->n_exc);
  memcpy(n->last_post, w + 4 + 2 * (size_t)n->n_exc, 4 * (size_t)n->n_exc);
  memcpy(n->last_pre, w + 4 + 3 * (size_t)n->n_exc, 4 * (size_t)n->n_in);
  return 0;
}

int oracle_get_stats(const oracle_net* n, uint64_t stats[8]) {
  if (!n || !stats) return E_INVAL;
  memcpy(stats, n->stats, sizeof(n->stats));
  return 0;
}

int oracle_q_max(const oracle_net* n) { return n ? n->q_max : E_INVAL; }

int oracle_lut(const oracle_net* n, int which, uint64_t* out, int cap) {
  if (!n || !out) return E_INVAL;
  int len; const uint64_t* src = NULL; const int64_t* srci = NULL;
  switch (which) {
    case 0: len = 256; src = n->thr_enc; break;
    case 1: len = n->L_pot; src = n->thr_pot; break;
    case 2: len = n->L_dep; src = n->thr_dep; break;
    case 3: len = n->q_max + 1; srci = n->det_p_base; break;
    case 4: len = n->q_max + 1; src = n->det_p_thr; break;
    case 5: len = n->q_max + 1; srci = n->det_d_base; break;
    case 6: len = n->q_max + 1; src = n->det_d_thr; break;
    default: return E_INVAL;
  }
  if (cap < len) return E_SIZE;
  for (int k = 0; k < len; ++k) out[k] = src ? src[k] : (uint64_t)srci[k];
  return len;
}

/* ---------------------------------------------------------------- NEXT-1: labelling + inference
 * P:88 §III-B: "After learning is complete, the first 1000 images in the test set are used to label all
 * the neurons in the first layer. The rest of the test set, which contains 9000 images, are used for
 * inference."  The labelling and voting rules are not stated; readings R21-R23. */
int oracle_infer(oracle_net* n, const uint8_t* images, int n_images, int T, const uint64_t* seeds,
                 uint32_t* counts) {
  if (!n || n_images < 0 || T < 0 || (n_images > 0 && (!images || !seeds || !counts))) return E_INVAL;
  const int we = (n->n_exc + 31) / 32;
  for (int k = 0; k < n_images; ++k) {
    int rc = oracle_present_ex(n, images + (size_t)k * n->n_in, T, seeds[k], ORACLE_NO_LEARN, 0);
    if (rc) return rc;
    for (int j = 0; j < n->n_exc; ++j) {
      uint32_t c = 0;
      for (int t = 0; t < T; ++t) c += (n->raster[(size_t)t * we + j / 32] >> (j % 32)) & 1u;
      counts[(size_t)k * n->n_exc + j] = c;
    }
  }
  return 0;
}

/* r_a / n_a > r_b / n_b, exactly (n_a, n_b > 0) */
static int ratio_gt(uint64_t r_a, uint64_t n_a, uint64_t r_b, uint64_t n_b) {
  return (unsigned __int128)r_a * n_b > (unsigned __int128)r_b * n_a;
}

int oracle_label(const uint32_t* counts, int n_images, int n_exc, const int32_t* classes, int n_classes,
                 int32_t* labels) {
  if (!counts || !classes || !labels || n_images < 0 || n_exc < 1 || n_classes < 1) return E_INVAL;
  uint64_t* N = (uint64_t*)calloc((size_t)n_classes, sizeof(uint64_t));
  uint64_t* r = (uint64_t*)calloc((size_t)n_classes, sizeof(uint64_t));
  if (!N || !r) { free(N); free(r); return E_NOMEM; }
  for (int k = 0; k < n_images; ++k) {
    if (classes[k] < 0 || classes[k] >= n_classes) { free(N); free(r); return E_INVAL; }
    N[classes[k]]++;
  }
  for (int j = 0; j < n_exc; ++j) {
    for (int c = 0; c < n_classes; ++c) r[c] = 0;
    for (int k = 0; k < n_images; ++k) r[classes[k]] += counts[(size_t)k * n_exc + j];
    int best = -1;
    for (int c = 0; c < n_classes; ++c) {
      if (N[c] == 0 || r[c] == 0) continue;            /* no response to class c */
      if (best < 0 || ratio_gt(r[c], N[c], r[best], N[best])) best = c;
    }
    labels[j] = best;
  }
  free(N); free(r);
  return 0;
}

int oracle_classify(const uint32_t* counts, int n_images, int n_exc, const int32_t* labels, int n_classes,
                    int32_t* pred) {
  if (!counts || !labels || !pred || n_images < 0 || n_exc < 1 || n_classes < 1) return E_INVAL;
  uint64_t* M = (uint64_t*)calloc((size_t)n_classes, sizeof(uint64_t));
  uint64_t* s = (uint64_t*)calloc((size_t)n_classes, sizeof(uint64_t));
  if (!M || !s) { free(M); free(s); return E_NOMEM; }
  for (int j = 0; j < n_exc; ++j) {
    if (labels[j] >= n_classes || labels[j] < -1) { free(M); free(s); return E_INVAL; }
    if (labels[j] >= 0) M[labels[j]]++;
  }
  for (int k = 0; k < n_images; ++k) {
    for (int c = 0; c < n_classes; ++c) s[c] = 0;
    for (int j = 0; j < n_exc; ++j)
      if (labels[j] >= 0) s[labels[j]] += counts[(size_t)k * n_exc + j];
    int best = -1;
    for (int c = 0; c < n_classes; ++c) {
      if (M[c] == 0 || s[c] == 0) continue;
      if (best < 0 || ratio_gt(s[c], M[c], s[best], M[best])) best = c;
    }
    pred[k] = best;
  }
  free(M); free(s);
  return 0;
}

/* ---------------------------------------------------------------- NEXT-4: Fig. 4 sparse workload
 * P:92 §IV-A: "We first evaluate the accuracy of the spiking neuron simulation (no learning) considering an
 * SNN of 10^3 LIF neurons and 10^4 synapses."  Topology, drive and delays are unstated: R24-R26. */
int oracle_sparse_run(const oracle_net* n, int n_in, int n_lif, const int32_t* src_off, const uint16_t* tgt,
                      const uint8_t* q, const uint8_t* images, int n_trials, int T, const uint64_t* seeds,
                      uint32_t* counts, uint32_t* raster) {
  if (!n || n_in < 1 || n_lif < 1 || n_lif > 65536 || !src_off || n_trials < 0 || T < 0) return E_INVAL;
  if (n_trials > 0 && (!images || !seeds || !counts)) return E_INVAL;
  const int n_src = n_in + n_lif;
  if (src_off[0] != 0) return E_INVAL;
  for (int s = 0; s < n_src; ++s) if (src_off[s + 1] < src_off[s]) return E_INVAL;
  const int n_syn = src_off[n_src];
  for (int k = 0; k < n_syn; ++k) if (tgt[k] >= n_lif || q[k] > n->q_max) return E_INVAL;
  const oracle_params* p = &n->p;
  const int fixed = p->membrane_mode == 1;
  const int wl = (n_lif + 31) / 32;
  float* vf = (float*)malloc(sizeof(float) * (size_t)n_lif);
  int32_t* vx = (int32_t*)malloc(sizeof(int32_t) * (size_t)n_lif);
  int32_t* cnt = (int32_t*)malloc(sizeof(int32_t) * (size_t)n_lif);
  int32_t* S = (int32_t*)malloc(sizeof(int32_t) * (size_t)n_lif);
  uint8_t* act = (uint8_t*)malloc((size_t)n_src);          /* source active at this step */
  uint8_t* spk = (uint8_t*)malloc((size_t)n_lif);          /* neuron spiked at this step */
  if (!vf || !vx || !cnt || !S || !act || !spk) { free(vf); free(vx); free(cnt); free(S); free(act); free(spk); return E_NOMEM; }
  for (int tr = 0; tr < n_trials; ++tr) {
    const uint8_t* img = images + (size_t)tr * n_in;
    for (int j = 0; j < n_lif; ++j) { vf[j] = n->vinitf; vx[j] = n->Vinit; cnt[j] = 0; spk[j] = 0; }   /* [R5] */
    for (int j = 0; j < n_lif; ++j) counts[(size_t)tr * n_lif + j] = 0;
    for (int t = 0; t < T; ++t) {
      /* sources: input pixels (encoder, R8, R13) at t; neurons that spiked at t-1 (one-step delay, R25) */
      for (int i = 0; i < n_in; ++i) {
        uint32_t u = draw(seeds[tr], (uint32_t)t, (uint32_t)(i >> 2), 0u, TAG_ENC, i & 3);
        act[i] = (uint8_t)((uint64_t)u < n->thr_enc[img[i]]);
      }
      for (int j = 0; j < n_lif; ++j) act[n_in + j] = spk[j];
      /* eq.(3) over the synapses of active sources */
      for (int j = 0; j < n_lif; ++j) S[j] = 0;
      for (int s = 0; s < n_src; ++s)
        if (act[s])
          for (int k = src_off[s]; k < src_off[s + 1]; ++k) S[tgt[k]] += q[k];
      /* eqs.(1)(2) + refractory [R6]; no inhibition, no WTA [R26] */
      for (int j = 0; j < n_lif; ++j) {
        spk[j] = 0;
        if (cnt[j] > 0) { cnt[j]--; continue; }
        int cross;
        if (fixed) { vx[j] = oracle_lif_step_fixed(n, vx[j], S[j]); cross = vx[j] > n->Vth; }
        else       { vf[j] = oracle_lif_step_fp32(n, vf[j], S[j]);  cross = vf[j] > n->vthf; }
        if (cross) {
          spk[j] = 1;
          vf[j] = n->vresetf; vx[j] = n->Vreset; cnt[j] = p->t_ref_steps;
          counts[(size_t)tr * n_lif + j]++;
          if (raster) raster[((size_t)tr * T + t) * wl + j / 32] |= 1u << (j % 32);
        }
      }
    }
  }
  free(vf); free(vx); free(cnt); free(S); free(act); free(spk);
  return 0;
}
