/*
 * hmg.h -- C ABI of the B200 (sm_100a) hmmsearch hot path: HMMER 3.0 MSV filter
 * and Viterbi filter (P7Viterbi with Lazy-F) scoring one profile HMM against
 * every sequence of a protein database.
 *
 * Paper: Jiang & Ganesan, "Fine-Grained Acceleration of HMMER 3.0 via
 * Architecture-aware Optimization on Massively Parallel Processors", IPDPSW
 * 2015.  "P:NNN" cites a line of the paper text.  The problem is
 * stated at P:21-23 / P:46-53 (score each target sequence against a query
 * profile, MSV then P7Viterbi, pass sequences by P-value threshold), Alg 1
 * (MSV) and Alg 2 (P7Viterbi).  Where the paper is
 * silent the HMMER 3.0 reading in DESIGN.md ("Readings", R1-R35) applies.
 *
 * Conventions (all entry points):
 *   - Plain C, no exceptions; every failure is a status code and leaves no
 *     side effect (outputs untouched, no handle created).
 *   - "host" pointers are CPU memory; "device" pointers are CUDA global memory
 *     on the handle's device.  Ownership of caller buffers never transfers.
 *   - Compute calls are asynchronous and stream-ordered on `stream`
 *     (a cudaStream_t passed as void*, NULL = legacy default stream).  They
 *     return after enqueueing; CUDA launch errors map to HMG_ECUDA.
 *   - Handles are immutable after creation (the per-F threshold tables a
 *     profile builds on first use are added under a lock and never freed or
 *     replaced before hmg_profile_destroy, so calls on other streams and CUDA
 *     graphs that captured them stay valid) and may be used from several
 *     streams; one handle must not be destroyed while work using it is in
 *     flight.
 *   - Sequence indices ("caller order") are positions 0..nseq-1 in the arrays
 *     given to hmg_db_create.  The DB is internally sorted by length
 *     (descending) for scheduling; all outputs are in caller order.
 *   - Overflow is a value, not an error: raw MSV 255 / raw Viterbi 32767 mean
 *     "score saturated" (+inf nats, P-value 0, always passes; reading R13/R17).
 *
 * Residue alphabet (Fig 6): codes 0..28 in the order
 *   A C D E F G H I K L M N P Q R S T V W Y - B J Z O U X * ~
 */
#ifndef HMG_H
#define HMG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  HMG_OK = 0,
  HMG_EINVAL = 1,        /* invalid argument (range, NaN, NULL, residue code > 28) */
  HMG_ENOMEM = 2,        /* host or device allocation failed */
  HMG_ECUDA = 3,         /* CUDA runtime / launch error (cudaGetLastError cleared) */
  HMG_EUNSUPPORTED = 4   /* valid but not supported (e.g. no sm_100 device) */
} hmg_status;

typedef struct hmg_profile hmg_profile; /* quantised profile, host + device tables */
typedef struct hmg_db hmg_db;           /* packed, length-sorted DB shard on one device */

/* Gumbel parameters of the two filter score distributions, in bits (P:41-45:
 * Viterbi/MSV high scores are Gumbel with lambda = log 2). */
typedef struct {
  double mu_msv, lambda_msv;
  double mu_vit, lambda_vit;
} hmg_evparams;

/* Quantised constants (read-only view for tests and score conversion). */
typedef struct {
  int M;
  int bias_b, tbm_b, tec_b, base_b; /* MSV byte system (Alg 1 l.15) */
  float scale_b;                    /* 3/ln2 (third-bits) */
  int base_w, xw_e, ddbound_w;      /* Viterbi word system (Alg 2 l.9) */
  float scale_w;                    /* 500/ln2 */
  const uint8_t* cost;              /* host [29][M]  biased byte costs, 255 = -inf */
  const int16_t* rsc;               /* host [29][M]  word emission scores */
  const int16_t* tsc;               /* host [8][M]   BM MM IM DM MD MI II DD (clamped) */
  int msv_fast;                     /* 1: exact fast MSV kernel applies (bias < 66 + tbm) */
  int msv_lanes, msv_regs;          /* MSV kernel geometry: lanes per sequence G, s16x2 regs Q */
  int vit_lanes, vit_nodes;         /* Viterbi s32 kernel geometry: lanes per sequence, nodes per lane */
  int vit_pair_lanes, vit_pair_regs; /* s16x2 pair Viterbi kernel (two cells per register) in front of
                                        the s32 kernel: lanes per sequence G, s16x2 registers Q per
                                        cell type; 0 = not used for this profile */
  int fwd_warps, fwd_nodes;         /* Forward kernel geometry: warps per sequence W, nodes per thread Q
                                       (Q = 16 up to 8 warps, else 8; 0 = no Forward stage: no tsc,
                                       or M > 4096) */
  int fwd_rows_smem;                /* emission-odds rows staged in shared memory (the rest via L1) */
  int fwd_seqs_per_block;           /* Forward kernel: sequences per block sharing the staged table */
  int fwd_lanes;                    /* Forward kernel: threads per sequence (8 = sub-warp lane groups
                                       for M <= 32; else 32 x fwd_warps) */
  int vit_pair_kernel;              /* which s16x2 Viterbi kernel (DESIGN.md 4.3b-d): 0 none, 1 lane groups
                                       (vit_pair), 2 warps joined per row (vit_cpair), 3 two warps
                                       without a row barrier (vit_cpair2), 4 one warp with the
                                       transitions in shared memory (vit_wide), 5 one warp with the
                                       transitions in tensor memory (vit_wide, tcgen05.ld) */
} hmg_quant;

/* ---------------------------------------------------------------- profile */

/* Load and quantise a profile (Alg 1 l.15 P:638; Alg 2 l.15-17 P:687-691).
 *   M    : model length, 1 <= M <= 100000.
 *   msc  : host float32 [M][29], match emission log-odds in nats; -INFINITY allowed,
 *          NaN / +INFINITY rejected.
 *   tsc  : host float32 [M][8], transition log-probabilities in nats (<= 0 or
 *          -INFINITY), per node k = 1..M (row k-1):
 *            0 BM  B->M_k        1 MM  M_{k-1}->M_k   2 IM  I_{k-1}->M_k   3 DM  D_{k-1}->M_k
 *            4 MD  M_k->D_{k+1}  5 MI  M_k->I_k       6 II  I_k->I_k       7 DD  D_k->D_{k+1}
 *          Nonexistent transitions (into node 1 from node 0, out of node M) are -INFINITY.
 *          May be NULL: then only the MSV filter is available.
 *   ev   : Gumbel parameters for pass flags; may be NULL if no pass flags are requested.
 *   device : CUDA device ordinal that receives the device tables; device < 0
 *          makes a host-only handle (quantised tables only; compute calls
 *          reject it) -- used to inspect the quantiser without a GPU.
 * Returns HMG_EINVAL on bad M / NaN / +inf / tsc > 0, HMG_ENOMEM, HMG_ECUDA. */
hmg_status hmg_profile_create(int M, const float* msc, const float* tsc, const hmg_evparams* ev,
                              int device, hmg_profile** out);

/* Fill *out with the quantised constants; the table pointers stay owned by the profile. */
hmg_status hmg_profile_quant(const hmg_profile* p, hmg_quant* out);

void hmg_profile_destroy(hmg_profile* p);

/* Gumbel locations of the MSV and Viterbi-filter score tails (high scores of the
 * optimal-alignment filters are Gumbel with lambda = log 2) for this profile, fitted on n
 * seeded background sequences of length L (HMMER3 amino background, 0.05% X) that the library
 * scores on the profile's device with its own kernels: mu = -ln(mean(exp(-lambda * bits)))/lambda,
 * the closed-form ML location for known lambda.  Fills out (mu_*, lambda_* = lambda).
 * Needs a device profile with tsc; n >= 1, L >= 1, lambda > 0.  Synchronous.  Profiles are
 * immutable: create the searching profile with the returned parameters. */
hmg_status hmg_calibrate(const hmg_profile* p, int n, int L, uint64_t seed, double lambda, hmg_evparams* out);

/* The same fit over a caller-supplied background database: every sequence of db is
 * scored with the library's MSV and Viterbi-filter kernels on the profile's device, converted to
 * bits with its own length (nats as hmg_msv_nats / hmg_vit_nats, null1 of its L), and
 * mu = -ln(mean over finite scores of exp(-lambda * bits)) / lambda.  hmg_calibrate is this call
 * on its generated sample.  db must live on the profile's device and hold >= 1 sequence; lambda
 * > 0; the profile needs tsc.  Synchronous.  HMG_EINVAL on bad arguments, HMG_ECUDA. */
hmg_status hmg_calibrate_db(const hmg_profile* p, const hmg_db* db, double lambda, hmg_evparams* out);


/* ---------------------------------------------------------------- database */

/* Pack a database and upload it to `device` (P:417-426 residue packing, Fig 6).
 *   dsq  : host uint8, all sequences concatenated, codes 0..28.
 *   off  : host int64 [nseq+1], sequence s is dsq[off[s] .. off[s+1]); lengths >= 1.
 *   nseq : >= 0.
 * Sequences are sorted by length (descending, stable), packed 6 residues per
 * 32-bit word (residue j of a word in bits [5j, 5j+5), bits 30-31 zero, unused
 * slots 31), each sequence starting on a 16-byte boundary.  device < 0 keeps
 * the packed image on the host only (inspection without a GPU). */
hmg_status hmg_db_create(const uint8_t* dsq, const int64_t* off, int64_t nseq, int device, hmg_db** out);

int64_t hmg_db_nseq(const hmg_db* db);
int64_t hmg_db_residues(const hmg_db* db);
int64_t hmg_db_packed_bytes(const hmg_db* db);   /* size of the packed residue image */

/* Long-sequence lane of this DB: the number of sequences (the longest, L > max(1500, 8 x mean
 * length)) that hmg_msv / hmg_pipeline score as parallel row chunks and, in the pipeline, on
 * SMs of their own; *residues (may be NULL) receives their residue count. */
int64_t hmg_db_long_lane(const hmg_db* db, int64_t* residues);

/* Host copy of the schedule: order[j] = caller index of the j-th sequence in
 * length-descending order (host int32 [nseq]). */
hmg_status hmg_db_order(const hmg_db* db, int32_t* order);

/* Host copy of the packed residue image (host uint32 [packed_bytes/4]); with
 * hmg_db_upload it lets a caller keep the image in pinned host memory and
 * re-send it (end-to-end timing: H2D of the DB inside the timed region). */
hmg_status hmg_db_image(const hmg_db* db, uint32_t* image);

/* Asynchronously re-upload the packed image (host, ideally pinned) into the DB's
 * device buffer on `stream`.  The image must come from hmg_db_image of this DB. */
hmg_status hmg_db_upload(hmg_db* db, const uint32_t* image, void* stream);

void hmg_db_destroy(hmg_db* db);

/* ---------------------------------------------------------------- filters */

/* MSV filter over every sequence (Alg 1).
 *   raw  : device uint8 [nseq], caller order: raw xJ, 255 = overflow.
 *   pass : device uint8 [nseq] or NULL: 1 iff P_msv <= F1 (needs ev; F1 in (0, 1]).
 * HMG_EINVAL if a pass buffer is given without ev, or F1 out of range. */
hmg_status hmg_msv(const hmg_profile* p, const hmg_db* db, double F1, void* stream, uint8_t* raw,
                   uint8_t* pass);

/* Viterbi filter (Alg 2; D->D by warp-synchronous Lazy-F) over the
 * n sequences listed in `ids` (device int32, caller order indices, may repeat).
 *   raw  : device int16 [nseq]; written only at the listed indices: raw xC,
 *          32767 = overflow, -32768 = -inf.
 *   pass : device uint8 [nseq] or NULL: written at the listed indices, 1 iff P_vit <= F2.
 * ids == NULL means all sequences (n ignored). */
hmg_status hmg_viterbi(const hmg_profile* p, const hmg_db* db, const int32_t* ids, int64_t n, double F2,
                       void* stream, int16_t* raw, uint8_t* pass);

/* The hmmsearch filter pipeline (Fig 1): MSV over all sequences ->
 * pass flags -> on-device stable compaction of survivors -> Viterbi filter over
 * the survivors only.  All outputs are device buffers in caller order:
 *   msv_raw      uint8 [nseq]
 *   vit_raw      int16 [nseq]  (written for survivors only)
 *   flags        uint8 [nseq]  bit0 MSV pass, bit1 Viterbi pass, bit2 Viterbi was run
 *   survivor_ids int32 [nseq]  caller indices of MSV survivors, length-descending order
 *   n_survivors  int64 [1]     device count of survivor_ids
 * Requires ev and tsc. */
hmg_status hmg_pipeline(const hmg_profile* p, const hmg_db* db, double F1, double F2, void* stream,
                        uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags, int32_t* survivor_ids,
                        int64_t* n_survivors);

/* Forward stage (Fig 1, the filter after P7Viterbi; "total
 * log-likelihood ratios summed over all possible alignments") over the n sequences
 * listed in `ids` (device int32, caller order; NULL = all sequences, n ignored).
 * Model: the same Plan-7 local multihit profile, in float32 odds space (emission odds
 * exp(msc), transition odds exp(tsc), exits M_k/D_k -> E = 1, E -> J = E -> C = 1/2, length
 * model N->N = J->J = C->C = L/(L+3), N->B = J->B = C->T = 3/(L+3); readings F1-F5),
 * rows rescaled by exact powers of two.
 *   nats : device float32 [nseq], written at the listed indices: the Forward score in nats
 *          (log of the summed path odds; -INFINITY if no path has non-zero odds).
 * Accuracy: float32 rounding, |error| <= 2^-24 (40 L + 4 M) + 1e-6 nats against exact arithmetic
 * on the paths that carry the score.  Needs tsc; HMG_EUNSUPPORTED for M > 4096
 * or emission log-odds above +40 nats (odds-space range). */
hmg_status hmg_forward(const hmg_profile* p, const hmg_db* db, const int32_t* ids, int64_t n, void* stream,
                       float* nats);

/* hmg_pipeline followed by the Forward stage on the sequences that passed the Viterbi filter
 * (Fig 1: MSV -> P7Viterbi -> Forward).  Outputs of hmg_pipeline, plus:
 *   fwd_nats  float32 [nseq]  Forward score (nats) of the Viterbi passes, written at those only
 *   fwd_ids   int32 [nseq]    caller indices of the Viterbi passes, length-descending order
 *   n_fwd     int64 [1]       device count of fwd_ids
 * and flags bit3 = the Forward stage ran for this sequence. */
hmg_status hmg_pipeline_forward(const hmg_profile* p, const hmg_db* db, double F1, double F2, void* stream,
                                uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags, int32_t* survivor_ids,
                                int64_t* n_survivors, float* fwd_nats, int32_t* fwd_ids, int64_t* n_fwd);

/* Many-profile MSV (the hmmscan / Pfam-scale workload): every
 * (profile, sequence) pair of nprof profiles x the DB in one call, one kernel launch per bucket of
 * profiles with a shared lane geometry (profiles padded to the bucket's largest model, <= 20%
 * padding).  Work items are (DB chunk, profile) in chunk-major order, so the longest sequences of
 * every profile start first and a chunk's residues stay in L2 while all profiles read them.
 *   profs : host array [nprof] of profiles on the DB's device (1 <= nprof <= 65535; repeats allowed).
 *   raw   : device uint8 [nprof][nseq], row i = profs[i], caller order: raw xJ as hmg_msv.
 *   pass  : device uint8 [nprof][nseq] or NULL: 1 iff P_msv <= F1 (every profile needs ev).
 * Results are identical to nprof hmg_msv calls (exact integer DP). */
hmg_status hmg_msv_batch(const hmg_profile* const* profs, int nprof, const hmg_db* db, double F1, void* stream,
                         uint8_t* raw, uint8_t* pass);

/* The Fig 1 filter pipeline for every profile of a batch: hmg_msv_batch's MSV stage, then per
 * profile (concurrently on side streams) pass flags + stable survivor compaction + the Viterbi
 * filter on its survivors.  Outputs are hmg_pipeline's, one row per profile (row i = profs[i]):
 *   msv_raw uint8 [nprof][nseq], vit_raw int16 [nprof][nseq] (survivors only), flags uint8
 *   [nprof][nseq], survivor_ids int32 [nprof][nseq] (row i holds n_survivors[i] caller indices,
 *   length-descending), n_survivors int64 [nprof] (device).
 * Optional Forward stage (all three NULL = off): fwd_nats float32 [nprof][nseq], fwd_ids int32
 * [nprof][nseq], n_fwd int64 [nprof] as hmg_pipeline_forward per row (flags bit3).
 * Every profile needs tsc and ev.  Results equal nprof hmg_pipeline (_forward) calls. */
hmg_status hmg_pipeline_batch(const hmg_profile* const* profs, int nprof, const hmg_db* db, double F1, double F2,
                              void* stream, uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags,
                              int32_t* survivor_ids, int64_t* n_survivors, float* fwd_nats, int32_t* fwd_ids,
                              int64_t* n_fwd);

/* Pass thresholds (reading R25) are integer tables by target length, built on the
 * host from the profile's Gumbel parameters per F.  A compute call builds the tables it needs on
 * first use (host binary search, cudaMalloc + cudaMemcpy: not allowed inside CUDA stream capture,
 * where such a call returns HMG_EUNSUPPORTED and leaves the capture intact).  This call builds them
 * ahead for MSV threshold F1 and Viterbi threshold F2 and target lengths up to Lmax (at least
 * 40000), so that a later call -- e.g. one captured in a CUDA graph -- finds them.  Tables stay
 * allocated until hmg_profile_destroy (graphs and other streams may hold them).
 * Needs a device profile with ev; F in (0, 1]; Lmax >= 1. */
hmg_status hmg_prepare_thresholds(const hmg_profile* p, double F1, double F2, int Lmax);

/* ---------------------------------------------------------------- tuning (performance only) */

/* Process-wide overrides of the kernel-geometry and schedule choices (the
 * defaults are the measured ones).  The library never reads the environment: results never depend
 * on these knobs (every kernel is exact), only performance does, and tests / sweeps set them here.
 * Knobs (int): MSV_G, VIT_G, MSV_LLONG, NO_LONG_LANE, FWD_QMAX, FWD_W, FWD_S, VIT_CTA, VIT_CTA_W,
 * VIT_GENERIC, NO_VIT_PAIR, VIT_PAIR_G, VIT_PAIR_CTA, VIT_SCAN, VIT_PAIR_W, VIT_PAIR_SG,
 * VIT_CPAIR2, LONG_S32, PIPE_LLONG, PIPE_CHUNK, UPLOAD_PARTS, UPLOAD_FIRST_PERMILLE, UPLOAD_GROW,
 * PIPE_LONG_SMS, MSV_BATCH_PAD, MSV_BATCH_ROUNDS, VIT_WIDE (0 off, 1 shared, 2 tensor memory),
 * LONG_PAIR_SMALL (0: models of <= 128 nodes keep the s32 long lane), UPLOAD_MSV_STREAMS.
 * Geometry knobs take effect at profile / DB
 * creation, schedule knobs at the next call.  HMG_EINVAL for an unknown name. */
hmg_status hmg_set_tuning(const char* name, int value);
/* Remove one override (name) or all of them (name == NULL). */
hmg_status hmg_clear_tuning(const char* name);

/* ---------------------------------------------------------------- instrumentation */

/* Number of CUDA kernels this library has launched since it was loaded. */
int64_t hmg_kernel_launches(void);

/* Stage timing (profiling aid, off by default).  When enabled, hmg_msv /
 * hmg_viterbi / hmg_pipeline / hmg_forward / hmg_pipeline_forward record CUDA events on their
 * stream between stages; hmg_stage_times waits for the last recorded event and fills
 * ms[6] with the durations of the most recent call's stages (-1 = not run):
 *   0 MSV fast kernel   1 MSV exact re-scoring (select + kernel)
 *   2 MSV pass flags + survivor compaction   3 Viterbi kernel   4 Viterbi flags/scatter
 *   5 Viterbi-pass compaction + Forward kernel
 * Not thread-safe across concurrent calls (one global set of events). */
hmg_status hmg_set_stage_timing(int enable);
hmg_status hmg_stage_times(double* ms);
/* With stage timing on: counts[0] = sequences of the most recent Viterbi stage that the s16x2
 * pair kernel handed to the s32 kernel (outside its 16-bit window: strong hits, overflow
 * neighbourhoods, all -inf rows), -1 if the pair kernel did not run.  Waits like hmg_stage_times. */
hmg_status hmg_stage_counts(int64_t* counts);

/* hmg_db_upload + hmg_pipeline with the upload overlapped: the packed image (host, pinned; from
 * hmg_db_image of this DB) is copied in length-ordered parts on a side stream (a first part of
 * 5% of the residues, then 4 parts of about equal residues; tuning knobs UPLOAD_PARTS /
 * UPLOAD_FIRST_PERMILLE / UPLOAD_GROW, hmg_set_tuning), each part's landing recorded as an event;
 * one MSV launch per part waits for its part's event only, the parts' launches rotating over two
 * side streams (UPLOAD_MSV_STREAMS) so each starts on the SMs the previous one's tail frees (the
 * long lane starts after the first part): the H2D of the later parts hides behind the filter of
 * the earlier ones.
 * Outputs and results are hmg_pipeline's.  The image must stay valid until the call's work on
 * `stream` has completed. */
hmg_status hmg_pipeline_upload(const hmg_profile* p, hmg_db* db, const uint32_t* image, double F1, double F2,
                               void* stream, uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags,
                               int32_t* survivor_ids, int64_t* n_survivors);

/* ---------------------------------------------------------------- host helpers (pure) */

/* Raw score -> nats for a length-L target ("Ensure ... (in nats)").
 * MSV: ((raw - tjb(L)) - 190)/scale_b - 3, +INF for 255.
 * VF : (raw + move(L) - 12000)/scale_w - 3, +INF for 32767, -INF for -32768. */
float hmg_msv_nats(int raw, int L);
float hmg_vit_nats(int raw, int L);
float hmg_null1_nats(int L);                               /* HMMER null1 (reading R24) */
double hmg_gumbel_surv(double bits, double mu, double lambda);
const char* hmg_strerror(hmg_status s);

#ifdef __cplusplus
}
#endif
#endif /* HMG_H */
