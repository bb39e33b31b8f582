/*
 * hmg_oracle.c -- plain, slow, obviously-correct CPU oracle for the hmmsearch
 * hot path of Jiang & Ganesan, "Fine-Grained Acceleration of HMMER 3.0 via
 * Architecture-aware Optimization on Massively Parallel Processors"
 * (IPDPSW 2015).  Citations "P:NNN" are lines of the paper text.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this file's
 * shared library.  It shares no code, header, table or constant generator
 * with the CUDA library under paper_conf_ipps_jiangg15_b200/csrc, and it
 * never includes anything from there.
 *
 * What it computes, in the paper's order:
 *   1. profile quantisation (HMMER 3.0 byte / word score systems; the paper
 *      names the 8-bit saturating biased system, Alg 1 l.15 P:638,
 *      and the -32768 word init, Alg 2 l.9 P:674; constants are the HMMER 3.0
 *      reading, SURVEY c.1 / DESIGN.md readings R1-R6);
 *   2. MSV filter, Alg 1 as a scalar row-by-row DP with explicit
 *      u8 saturation after every operation;
 *   3. Viterbi filter, Alg 2 as a scalar DP with explicit s16
 *      saturation, the D->D chain resolved by the FULL sequential closure on
 *      every row (Lazy-F, P:519-533 / P:727-790, is an exact shortcut of this
 *      closure, so the oracle does not take it);
 *   4. score conversion to nats, null1, Gumbel survival and pass decisions
 *      (HMMER 3.0 pipeline reading, R9-R12);
 *   5. Forward score: "the total log-likelihood ratios summed
 *      over all possible alignments" of the same Plan-7 local
 *      multihit model (Fig 3), in double precision log space, the textbook
 *      Forward recurrence with HMMER 3.0's full length model (readings F1-F5 in
 *      DESIGN.md); the stage after P7Viterbi in Fig 1.
 *
 * Layouts (same meaning as include/hmg.h, restated, not shared):
 *   msc : float32 [M][29] log-odds in nats, residue order
 *         A C D E F G H I K L M N P Q R S T V W Y - B J Z O U X * ~  (codes 0..28)
 *   tsc : float32 [M][8]  per node k=1..M (row k-1):
 *         0 BM (B->M_k)  1 MM (M_{k-1}->M_k)  2 IM (I_{k-1}->M_k)  3 DM (D_{k-1}->M_k)
 *         4 MD (M_k->D_{k+1})  5 MI (M_k->I_k)  6 II (I_k->I_k)  7 DD (D_k->D_{k+1})
 *   dsq : uint8 residue codes 0..28, sequences concatenated, off[nseq+1] int64.
 *
 * Build: gcc -O2 -std=c11 -shared -fPIC -pthread -o liboracle.so hmg_oracle.c -lm
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_K 29          /* alphabet size incl. degenerate and gap codes */
#define OR_KCANON 20     /* canonical residues used for the byte bias */
#define OR_LN2 0.69314718055994529

/* ------------------------------------------------------------------------ */
/* 1. Quantisation (SURVEY c.1; R1-R6)                             */
/* ------------------------------------------------------------------------ */

static float or_scale_b(void) { return (float)(3.0 / OR_LN2); }   /* third-bits */
static float or_scale_w(void) { return (float)(500.0 / OR_LN2); } /* 1/500 bits */

/* Unbiased byte cost of a score s <= 0: -round(scale_b*s), capped at 255. */
int or_ub(float s) {
  float c = -1.0f * roundf(or_scale_b() * s);
  if (c > 255.0f) return 255;
  return (int)c;
}

/* Biased byte cost: -round(scale_b*s) + bias, 255 (= -inf) when it exceeds
 * 255 - bias.  A column above the canonical maximum (only possible for a
 * caller-built non-canonical column) would give a negative cost; it is floored
 * at 0 (reading R4). */
int or_bb(float s, int bias) {
  float c = -1.0f * roundf(or_scale_b() * s);
  if (c > (float)(255 - bias)) return 255;
  int v = (int)c + bias;
  return v < 0 ? 0 : v;
}

/* Word score: round(scale_w*s) clamped to [-32768, 32767]; -inf -> -32768. */
int or_w(float s) {
  float r = roundf(or_scale_w() * s);
  if (r >= 32767.0f) return 32767;
  if (r <= -32768.0f) return -32768;
  return (int)r;
}

int or_tjb_b(int L) { return or_ub(logf(3.0f / (float)(L + 3))); }
int or_move_w(int L) { return or_w(logf(3.0f / (float)(L + 3))); }
int or_tbm_b(int M) { return or_ub(logf(2.0f / ((float)M * (float)(M + 1)))); }
int or_tec_b(void) { return or_ub(logf(0.5f)); }
int or_xw_e(void) { return or_w(logf(0.5f)); }

/* MSV byte profile: fills cost[29][M] (row x, column k-1); returns the bias. */
int or_quant_msv(int M, const float* msc, uint8_t* cost, int* out_bias, int* out_tbm, int* out_tec) {
  float mx = 0.0f;
  for (int k = 0; k < M; ++k)
    for (int x = 0; x < OR_KCANON; ++x)
      if (msc[k * OR_K + x] > mx) mx = msc[k * OR_K + x];
  int bias = or_ub(-1.0f * mx);
  for (int x = 0; x < OR_K; ++x)
    for (int k = 0; k < M; ++k) cost[x * M + k] = (uint8_t)or_bb(msc[k * OR_K + x], bias);
  *out_bias = bias;
  *out_tbm = or_tbm_b(M);
  *out_tec = or_tec_b();
  return bias;
}

/* Viterbi word profile.  rsc is [29][M]; tr is [8][M] in the tsc order above,
 * clamped: BM,MM,IM,DM,MD,MI <= 0, II <= -1, DD unclamped (reading R6). */
int or_quant_vit(int M, const float* msc, const float* tsc, int16_t* rsc, int16_t* tr, int* out_ddbound) {
  for (int x = 0; x < OR_K; ++x)
    for (int k = 0; k < M; ++k) rsc[x * M + k] = (int16_t)or_w(msc[k * OR_K + x]);
  for (int t = 0; t < 8; ++t)
    for (int k = 0; k < M; ++k) {
      int v = or_w(tsc[k * 8 + t]);
      if (t <= 5 && v > 0) v = 0;
      if (t == 6 && v > -1) v = -1;
      tr[t * M + k] = (int16_t)v;
    }
  /* ddbound = max_{k=2..M-2} w(DD_k) + w(DM_{k+2}) - w(BM_{k+2}); -32768 if empty. */
  int ddb = -32768;
  for (int k = 2; k <= M - 2; ++k) {
    int v = or_w(tsc[(k - 1) * 8 + 7]) + or_w(tsc[(k + 1) * 8 + 3]) - or_w(tsc[(k + 1) * 8 + 0]);
    if (v > ddb) ddb = v;
  }
  *out_ddbound = ddb;
  return 0;
}

/* ------------------------------------------------------------------------ */
/* 2. MSV filter, Alg 1                                          */
/* ------------------------------------------------------------------------ */

static int sat_u8(int v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

/* Scalar MSV of one sequence.  Returns raw xJ (0..251-bias) or 255 on
 * overflow.  prev/cur are caller scratch of M+1 ints. */
static int or_msv_one(int M, const uint8_t* cost, int bias, int tbm, int tec, int tjb, const uint8_t* dsq, int L,
                      int* prev, int* cur) {
  const int base = 190;
  for (int k = 0; k <= M; ++k) prev[k] = 0;   /* Alg 1 l.9: mmx <- 0 (u8 -inf) */
  int xJ = 0;
  int xB = sat_u8(base - tjb);
  for (int i = 1; i <= L; ++i) {               /* Alg 1 l.10 row loop */
    int x = dsq[i - 1];                        /* l.11 decode residue */
    int xBp = sat_u8(xB - tbm);                /* B->M_k, uniform entry (reading R7) */
    int xE = 0;                                /* l.12 */
    cur[0] = 0;
    for (int k = 1; k <= M; ++k) {             /* l.14 */
      int s = prev[k - 1] > xBp ? prev[k - 1] : xBp;   /* l.15 max(mmx, xB) */
      s = sat_u8(s + bias);                            /*      + bias       */
      s = sat_u8(s - (int)cost[x * M + (k - 1)]);      /*      - em(res,p)  */
      cur[k] = s;
      if (s > xE) xE = s;                              /* l.16 */
    }
    if (xE >= 255 - bias) return 255;          /* overflow -> +inf (reading R13) */
    int e = sat_u8(xE - tec);                  /* l.20: E->J */
    if (e > xJ) xJ = e;
    xB = sat_u8((xJ > base ? xJ : base) - tjb);/*       J->B / N->B */
    int* t = prev; prev = cur; cur = t;
  }
  return xJ;                                   /* l.23 score(xJ) */
}

/* tjb < 0: take tjb_b(L) of the target length (the normal case); an explicit
 * tjb >= 0 fixes the length parameter (invariant tests append residues). */
int or_msv_seq(int M, const uint8_t* cost, int bias, int tbm, int tec, const uint8_t* dsq, int L, int tjb) {
  int* buf = (int*)malloc(sizeof(int) * 2 * (size_t)(M + 1));
  if (!buf) return -1;
  if (tjb < 0) tjb = or_tjb_b(L);
  int r = or_msv_one(M, cost, bias, tbm, tec, tjb, dsq, L, buf, buf + M + 1);
  free(buf);
  return r;
}

/* ------------------------------------------------------------------------ */
/* 3. Viterbi filter, Alg 2, full D->D closure per row            */
/* ------------------------------------------------------------------------ */

static int sat_s16(int v) { return v < -32768 ? -32768 : (v > 32767 ? 32767 : v); }

/* Returns raw xC (int16 range) or 32767 on overflow.  Scratch: 6*(M+1) ints. */
static int or_vit_one(int M, const int16_t* rsc, const int16_t* tr, const uint8_t* dsq, int L, int move, int* scratch) {
  int* Mp = scratch;            int* Ip = Mp + (M + 1); int* Dp = Ip + (M + 1);
  int* Mn = Dp + (M + 1);       int* In = Mn + (M + 1); int* Dn = In + (M + 1);
  const int16_t* tBM = tr + 0 * M; const int16_t* tMM = tr + 1 * M;
  const int16_t* tIM = tr + 2 * M; const int16_t* tDM = tr + 3 * M;
  const int16_t* tMD = tr + 4 * M; const int16_t* tMI = tr + 5 * M;
  const int16_t* tII = tr + 6 * M; const int16_t* tDD = tr + 7 * M;
  const int NEG = -32768;
  int xE_w = or_xw_e();                       /* E->C, E->J = log 0.5 (reading R9) */
  for (int k = 0; k <= M; ++k) Mp[k] = Ip[k] = Dp[k] = NEG;   /* Alg 2 l.9 */
  int xN = 12000;                             /* base_w */
  int xB = xN + move;
  int xJ = NEG, xC = NEG;
  for (int i = 1; i <= L; ++i) {
    int x = dsq[i - 1];
    int xE = NEG;
    Mn[0] = In[0] = Dn[0] = NEG;
    for (int k = 1; k <= M; ++k) {
      /* l.16 (+ emission, reading R15): M(i,k) */
      int b = sat_s16(xB + tBM[k - 1]);
      int mm = sat_s16(Mp[k - 1] + tMM[k - 1]);
      int im = sat_s16(Ip[k - 1] + tIM[k - 1]);
      int dm = sat_s16(Dp[k - 1] + tDM[k - 1]);
      int m = b;
      if (mm > m) m = mm;
      if (im > m) m = im;
      if (dm > m) m = dm;
      Mn[k] = sat_s16(m + rsc[x * M + (k - 1)]);
      /* l.15: I(i,k) */
      int mi = sat_s16(Mp[k] + tMI[k - 1]);
      int ii = sat_s16(Ip[k] + tII[k - 1]);
      In[k] = mi > ii ? mi : ii;
      /* l.17 partial D (reading R16: it belongs to node k+1) */
      Dn[k] = (k == 1) ? NEG : sat_s16(Mn[k - 1] + tMD[k - 2]);
      if (Mn[k] > xE) xE = Mn[k];             /* l.18 */
    }
    if (xE >= 32767) return 32767;            /* overflow -> +inf (reading R17) */
    /* l.24 specials */
    int e = xE + xE_w;
    if (e > xC) xC = e;
    if (e > xJ) xJ = e;
    xB = (xJ > xN ? xJ : xN) + move;
    /* l.25: the D->D chain.  Full sequential closure (Lazy-F is an exact
     * shortcut of exactly this). */
    for (int k = 2; k <= M; ++k) {
      int dd = sat_s16(Dn[k - 1] + tDD[k - 2]);
      if (dd > Dn[k]) Dn[k] = dd;
    }
    int* t;
    t = Mp; Mp = Mn; Mn = t;
    t = Ip; Ip = In; In = t;
    t = Dp; Dp = Dn; Dn = t;
  }
  return xC;                                   /* l.28 score(xC) */
}

/* move > 0: take move_w(L) of the target length; move <= 0 fixes it. */
int or_vit_seq(int M, const int16_t* rsc, const int16_t* tr, const uint8_t* dsq, int L, int move) {
  int* buf = (int*)malloc(sizeof(int) * 6 * (size_t)(M + 1));
  if (!buf) return -32769;
  if (move > 0) move = or_move_w(L);
  int r = or_vit_one(M, rsc, tr, dsq, L, move, buf);
  free(buf);
  return r;
}

/* ------------------------------------------------------------------------ */
/* Multi-threaded drivers over a database (timed as the CPU baseline)        */
/* ------------------------------------------------------------------------ */

typedef struct {
  int kind; /* 0 msv, 1 vit */
  int M;
  const uint8_t* cost; int bias, tbm, tec;
  const int16_t* rsc; const int16_t* tr;
  const uint8_t* dsq; const int64_t* off;
  const int64_t* ids; int64_t n;  /* which sequences (NULL = 0..n-1) */
  int* out;                       /* indexed like ids (position j) */
  int64_t next;                   /* shared work counter */
  pthread_mutex_t mu;
} or_job;

static void* or_worker(void* arg) {
  or_job* J = (or_job*)arg;
  int* scratch = (int*)malloc(sizeof(int) * 6 * (size_t)(J->M + 1));
  for (;;) {
    int64_t lo, hi;
    pthread_mutex_lock(&J->mu);
    lo = J->next; hi = lo + 16; if (hi > J->n) hi = J->n; J->next = hi;
    pthread_mutex_unlock(&J->mu);
    if (lo >= J->n) break;
    for (int64_t j = lo; j < hi; ++j) {
      int64_t s = J->ids ? J->ids[j] : j;
      const uint8_t* d = J->dsq + J->off[s];
      int L = (int)(J->off[s + 1] - J->off[s]);
      if (J->kind == 0)
        J->out[j] = or_msv_one(J->M, J->cost, J->bias, J->tbm, J->tec, or_tjb_b(L), d, L, scratch,
                               scratch + J->M + 1);
      else
        J->out[j] = or_vit_one(J->M, J->rsc, J->tr, d, L, or_move_w(L), scratch);
    }
  }
  free(scratch);
  return 0;
}

static void or_run(or_job* J, int nthreads) {
  if (nthreads < 1) nthreads = 1;
  pthread_mutex_init(&J->mu, 0);
  J->next = 0;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)nthreads);
  for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], 0, or_worker, J);
  for (int t = 0; t < nthreads; ++t) pthread_join(th[t], 0);
  free(th);
  pthread_mutex_destroy(&J->mu);
}

/* Score sequences ids[0..n) (or 0..n-1 when ids == NULL) of a concatenated DB. */
void or_msv_db(int M, const uint8_t* cost, int bias, int tbm, int tec, const uint8_t* dsq, const int64_t* off,
               const int64_t* ids, int64_t n, int nthreads, int* out) {
  or_job J; memset(&J, 0, sizeof J);
  J.kind = 0; J.M = M; J.cost = cost; J.bias = bias; J.tbm = tbm; J.tec = tec;
  J.dsq = dsq; J.off = off; J.ids = ids; J.n = n; J.out = out;
  or_run(&J, nthreads);
}

void or_vit_db(int M, const int16_t* rsc, const int16_t* tr, const uint8_t* dsq, const int64_t* off,
               const int64_t* ids, int64_t n, int nthreads, int* out) {
  or_job J; memset(&J, 0, sizeof J);
  J.kind = 1; J.M = M; J.rsc = rsc; J.tr = tr;
  J.dsq = dsq; J.off = off; J.ids = ids; J.n = n; J.out = out;
  or_run(&J, nthreads);
}

/* ------------------------------------------------------------------------ */
/* 4. Conversion, null model, Gumbel tail, pass decisions (R9-R12)  */
/* ------------------------------------------------------------------------ */

/* MSV nats: ((xJ - tjb) - base_b) / scale_b - 3 ; +inf for the overflow raw. */
float or_msv_nats(int raw, int L) {
  if (raw == 255) return INFINITY;
  float sc = ((float)(raw - or_tjb_b(L)) - 190.0f);
  sc /= or_scale_b();
  sc -= 3.0;
  return sc;
}

/* Viterbi-filter nats: (xC + move - base_w) / scale_w - 3 ; +inf overflow,
 * -inf when no path (xC = -32768). */
float or_vit_nats(int raw, int L) {
  if (raw == 32767) return INFINITY;
  if (raw == -32768) return -INFINITY;
  float sc = ((float)(raw + or_move_w(L)) - 12000.0f);
  sc /= or_scale_w();
  sc -= 3.0;
  return sc;
}

/* HMMER null1 of a length-L target: L*log(p1) + log(1-p1), p1 = L/(L+1). */
float or_null1(int L) {
  float p1 = (float)L / (float)(L + 1);
  return (float)((float)L * log((double)p1) + log(1.0 - (double)p1));
}

double or_gumbel_surv(double x, double mu, double lambda) {
  double y = lambda * (x - mu);
  double ey = -exp(-y);
  if (fabs(ey) < 5e-9) return -ey;
  return 1.0 - exp(ey);
}

/* P-value of a score in nats for a length-L target. */
double or_pvalue(float nats, int L, double mu, double lambda) {
  if (nats == INFINITY) return 0.0;
  if (nats == -INFINITY) return 1.0;
  double bits = (double)(nats - or_null1(L)) / OR_LN2;
  return or_gumbel_surv(bits, mu, lambda);
}

/* pass <=> not (P > F) (HMMER pipeline test). */
int or_msv_pass(int raw, int L, double mu, double lambda, double F) {
  return !(or_pvalue(or_msv_nats(raw, L), L, mu, lambda) > F);
}

int or_vit_pass(int raw, int L, double mu, double lambda, double F) {
  return !(or_pvalue(or_vit_nats(raw, L), L, mu, lambda) > F);
}

/* Bits score (for mu calibration): (nats - null1)/ln2. */
double or_bits(float nats, int L) { return (double)(nats - or_null1(L)) / OR_LN2; }

/* ------------------------------------------------------------------------ */
/* 5. Forward score (f2; "summed over all possible alignments",      */
/*    Fig 1; readings F1-F5)                                       */
/* ------------------------------------------------------------------------ */

static double or_lse(double a, double b) {            /* log(e^a + e^b), -inf aware */
  if (a == -INFINITY) return b;
  if (b == -INFINITY) return a;
  return a > b ? a + log1p(exp(b - a)) : b + log1p(exp(a - b));
}

/* Forward score in nats of one sequence: log of the summed odds of every path
 * S -> N* -> B -> (M|I|D)+ -> E -> (J -> B ...)* -> C* -> T, where
 *   emissions: M_k emits x with odds exp(msc[k][x]); I_k, N, C, J emit with odds 1 (F3, F4);
 *   transitions: the profile's tsc (log probabilities; -inf = absent), local entry
 *   B->M_k = tsc[k][BM], local exit M_k->E and D_k->E = 1 (F1), E->C = E->J = 1/2 (R9),
 *   length model N->N = J->J = C->C = L/(L+3), N->B = J->B = C->T = 3/(L+3) (F2).
 * Rows are computed in the paper's order (Alg 2's row loop, with sums in place of
 * maxima): M and I from row i-1, D along row i, then E, N, J, C, B (F5). */
double or_fwd_seq(int M, const float* msc, const float* tsc, const uint8_t* dsq, int L, double* scratch) {
  double* Mp = scratch;            double* Ip = Mp + (M + 1);   double* Dp = Ip + (M + 1);
  double* Mn = Dp + (M + 1);       double* In = Mn + (M + 1);   double* Dn = In + (M + 1);
  const double loop = log((double)L / (double)(L + 3)), move = log(3.0 / (double)(L + 3));
  const double half = log(0.5);
#define TS(k, t) ((double)tsc[(size_t)((k) - 1) * 8 + (t)])   /* node k = 1..M */
  for (int k = 0; k <= M; ++k) Mp[k] = Ip[k] = Dp[k] = -INFINITY;
  double N = 0.0, J = -INFINITY, C = -INFINITY, B = N + move;     /* row 0 */
  for (int i = 0; i < L; ++i) {
    const int x = dsq[i];
    Mn[0] = In[0] = Dn[0] = -INFINITY;
    for (int k = 1; k <= M; ++k) {
      double sm = B + TS(k, 0);                                      /* B -> M_k */
      if (k > 1) {
        sm = or_lse(sm, Mp[k - 1] + TS(k, 1));                       /* M_{k-1} -> M_k */
        sm = or_lse(sm, Ip[k - 1] + TS(k, 2));                       /* I_{k-1} -> M_k */
        sm = or_lse(sm, Dp[k - 1] + TS(k, 3));                       /* D_{k-1} -> M_k */
      }
      Mn[k] = sm + (double)msc[(size_t)(k - 1) * OR_K + x];
      In[k] = (k < M) ? or_lse(Mp[k] + TS(k, 5), Ip[k] + TS(k, 6)) : -INFINITY;   /* odds 1 */
      Dn[k] = (k > 1) ? or_lse(Mn[k - 1] + TS(k - 1, 4), Dn[k - 1] + TS(k - 1, 7)) : -INFINITY;
    }
    double E = -INFINITY;
    for (int k = 1; k <= M; ++k) E = or_lse(E, or_lse(Mn[k], Dn[k]));     /* M_k, D_k -> E */
    N = N + loop;
    J = or_lse(J + loop, E + half);
    C = or_lse(C + loop, E + half);
    B = or_lse(N + move, J + move);
    double* t;
    t = Mp; Mp = Mn; Mn = t;
    t = Ip; Ip = In; In = t;
    t = Dp; Dp = Dn; Dn = t;
  }
#undef TS
  return C + move;                                                    /* C -> T */
}

typedef struct {
  int M; const float* msc; const float* tsc;
  const uint8_t* dsq; const int64_t* off; const int64_t* ids; int64_t n;
  double* out; int64_t next; pthread_mutex_t mu;
} or_fjob;

static void* or_fworker(void* arg) {
  or_fjob* J = (or_fjob*)arg;
  double* scratch = (double*)malloc(sizeof(double) * 6 * (size_t)(J->M + 1));
  for (;;) {
    int64_t lo, hi;
    pthread_mutex_lock(&J->mu);
    lo = J->next; hi = lo + 4; if (hi > J->n) hi = J->n; J->next = hi;
    pthread_mutex_unlock(&J->mu);
    if (lo >= J->n) break;
    for (int64_t j = lo; j < hi; ++j) {
      int64_t s = J->ids ? J->ids[j] : j;
      J->out[j] = or_fwd_seq(J->M, J->msc, J->tsc, J->dsq + J->off[s], (int)(J->off[s + 1] - J->off[s]), scratch);
    }
  }
  free(scratch);
  return 0;
}

void or_fwd_db(int M, const float* msc, const float* tsc, const uint8_t* dsq, const int64_t* off,
               const int64_t* ids, int64_t n, int nthreads, double* out) {
  or_fjob J; memset(&J, 0, sizeof J);
  J.M = M; J.msc = msc; J.tsc = tsc; J.dsq = dsq; J.off = off; J.ids = ids; J.n = n; J.out = out;
  if (nthreads < 1) nthreads = 1;
  pthread_mutex_init(&J.mu, 0);
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)nthreads);
  for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], 0, or_fworker, &J);
  for (int t = 0; t < nthreads; ++t) pthread_join(th[t], 0);
  free(th);
  pthread_mutex_destroy(&J.mu);
}
