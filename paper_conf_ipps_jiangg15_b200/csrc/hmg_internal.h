// hmg_internal.h -- private structures of libhmg (host C++ and CUDA sides).
// Nothing here is shared with oracle/ (the CPU oracle is an independent program).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <mutex>
#include <vector>

#include "../../include/hmg.h"

namespace hmg {

constexpr int kAlpha = 29;      // 20 + 6 degenerate + 3 gap codes
constexpr int kRows = 32;       // profile rows in device tables: 29 codes + 3 pad rows (code 31 = pad)
constexpr int kPadCode = 31;    // unused slots of the last word are 31
constexpr int kBaseB = 190;     // MSV byte base (reading R1)
constexpr int kBaseW = 12000;   // Viterbi word base (reading R2)
constexpr int16_t kNegE = -16384;   // "minus infinity" emission / carry of the s16x2 MSV lanes
constexpr int kNegW = -32768;       // word -inf (Alg 2 l.9 P:674)

#ifdef MSV_NO_BYTE
constexpr bool kMsvByte = false;     // A/B builds: the 2-word remainder stays s16x2
#else
constexpr bool kMsvByte = true;
#endif
#ifdef MSV_Q_PLUS1
constexpr bool kMsvQPlus1 = true;    // A/B builds: 2GQ >= M + 1 (a successor cell for node M)
#else
constexpr bool kMsvQPlus1 = false;
#endif
// MsvLayout<G, Q> (msv.cuh) for run-time (G, Q): words per residue row (STRIDE), the offsets of the
// remainder chunks' copy 0 (b2, b1), their copy counts, and the table size in words (WORDS).
// The host table builder (host.cu msv_table) and the launchers use this; msv.cu checks it
// against the template for every instantiated geometry.
// byte: G = 8 / 16 with a 2-word remainder hold it as one word of four int8 emissions per lane
// (32 / G copies, widened by PRMT; valid when msv_byte_exact holds, else the exact kernel runs).
struct MsvLayoutRT {
  int n4, has2, has1, byte, nc2, nc1, b2, b1, roww, ncopy, stride, copy, words;
  __host__ __device__ constexpr MsvLayoutRT(int G, int Q)
      : n4(Q / 4), has2(Q % 4 >= 2), has1(Q % 2), byte(kMsvByte && (G == 8 || G == 16) && Q % 4 >= 2),
        nc2(G == 8 ? 2 : 1), nc1(G == 8 ? 4 : (G == 16 ? 2 : 1)),
        b2(Q / 4 * 4 * G), b1(Q / 4 * 4 * G + (Q % 4 >= 2 ? 2 * G * (G == 8 ? 2 : 1) : 0)),
        roww(Q / 4 * 4 * G + (Q % 4 >= 2 ? 2 * G * (G == 8 ? 2 : 1) : 0) +
             (Q % 2 ? G * (G == 8 ? 4 : (G == 16 ? 2 : 1)) : 0)),
        ncopy(G < 8 ? 8 / G : 1),
        stride(0), copy(0), words(0) {
    stride = ncopy > 1 ? (roww + 31) / 32 * 32 : roww;
    copy = kRows * stride;
    words = ((ncopy * copy + (ncopy - 1) * 4 * G) + 3) / 4 * 4;
  }
};

// int8 emissions (clamped at -128) are exact in the MSV fast kernel when every cell that takes an
// emission is at most 128 above B': cells stay below the J->B threshold, at most
// 3 + tjb + tbm (+ bias within a voting row) above B'.
__host__ __device__ constexpr bool msv_byte_exact(int tjb_max, int tbm, int bias) {
  return 3 + tjb_max + tbm + bias <= 128;
}

// ---------------------------------------------------------------- MSV kernel arguments

struct MsvArgs {
  const uint32_t* words;     // packed residues
  const uint32_t* woff16;    // [nseq] sorted: word offset / 4 (16-byte units)
  const int32_t* len;        // [nseq] sorted lengths (descending)
  int64_t nseq;
  int64_t nlong;             // fast kernel: the first nlong sorted sequences go to the G=32 queue
  int skip_long;             // 1: sequences [0, nlong) are scored elsewhere (pipeline long lane)
  const uint8_t* tjb;        // [Lmax+1] tjb_b(L)
  const uint32_t* prof;      // striped s16x2 emission table for (G, Q), kRows rows
  const uint8_t* cost;       // plain biased costs [kRows][M] (exact kernel)
  int M, bias, tbm;
  uint8_t* raw;              // [nseq] sorted order output
  unsigned long long* counter;  // work-queue counter, zero at launch
  const int32_t* list;       // exact kernel: sorted indices to redo
  const int64_t* nlist;      // exact kernel: device count
  uint8_t* scratch;          // exact kernel: per-warp row buffers
};

// Many-profile MSV (msv_multi.cuh): a bucket of profiles with one lane geometry
struct MsvMultiArgs {
  MsvArgs base;              // DB fields (words, woff16, len, nseq, tjb); bias/tbm/raw set per profile
  int nprof;
  const uint32_t* const* prof;  // [nprof] striped tables in the bucket's (G, Q) layout
  const int* bias;           // [nprof]
  const int* tbm;            // [nprof]
  uint8_t* raw;              // [nprof][nseq] sorted order (row p of the bucket)
  long long nchunks;
  int chunk;                 // sequences per chunk
  unsigned long long* counter;
};

// exact MSV over (profile, sequence) pairs (msv_multi.cu): list entry j = p * nseq + s
struct MsvPairArgs {
  const uint32_t* words;
  const uint32_t* woff16;
  const int32_t* len;
  int64_t nseq;
  const uint8_t* tjb;
  const uint8_t* const* cost;   // [nprof] plain biased costs [kRows][M_p]
  const int* M;
  const int* bias;
  const int* tbm;
  const int64_t* list;
  const int64_t* nlist;
  uint8_t* raw;              // [nprof][nseq] sorted order
  uint8_t* scratch;          // per-warp rows, 2 (Mmax + 1) bytes each
  int Mmax;
};

// ---------------------------------------------------------------- Viterbi kernel arguments
struct VitArgs {
  const uint32_t* words;
  const uint32_t* woff16;
  const int32_t* len;
  int64_t nseq;
  const int16_t* move;       // [Lmax+1] move_w(L)
  const int16_t* rsc;        // register kernel: striped [kRows][G][Q] s16 ; generic: plain [kRows][M]
  const int32_t* tr;         // register kernel: striped [8][G][Q] s32 ; generic: plain s32 [8][M]
  int M;
  const int32_t* list;       // sorted indices to score (NULL = all, in order)
  const int64_t* nlist;      // device count when list != NULL
  int16_t* raw_sorted;       // [nseq] output, sorted order
  unsigned long long* counter;
  int32_t* scratch;          // generic kernel: per-warp rows
  const uint8_t* done;       // skip sorted index s < ndone when done[s] (the pipeline long lane owns it)
  int64_t ndone;
  // s16x2 pair kernel (vit_pair.cuh): per-sequence floor F = sat16(12000 + move(L) + tbm_min),
  // safe = 32767 - (largest emission score); sequences outside the 16-bit window go to redo_list
  int tbm_min, safe;
  int32_t* redo_list;
  unsigned long long* redo_count;
};

// Long-sequence lane (long.cu): chunked whole-warp MSV for the longest sequences and, in the
// pipeline, whole-warp Viterbi for their MSV survivors on SMs held alone.
struct LongArgs {
  MsvArgs m;                 // m.prof = whole-warp MSV table (32, QL), m.raw = MSV raw (sorted)
  VitArgs v;                 // v.rsc / v.tr = register-kernel tables (32, QV), v.raw_sorted
  const uint16_t* thr;       // MSV pass threshold by length
  uint8_t* owned;            // [nlong] 1: the long lane runs the Viterbi filter of this sequence
  int64_t nlong;
  const int32_t* chunk_start;  // [nlong+1] exclusive prefix of row chunks per long sequence
  int64_t nitems;            // total chunks
  int chunk_rows;
  int* chunk_max;            // [nitems]
  unsigned* chunk_done;      // [nlong] chunks finished
  unsigned long long* counter;  // [2] work queues (chunks, Viterbi)
};

// Forward filter stage (forward.cu): float odds-space Forward over a sorted list
struct FwdArgs {
  const uint32_t* words;
  const uint32_t* woff16;
  const int32_t* len;
  const int32_t* order;        // sorted -> caller
  const int32_t* list;         // sorted indices (NULL = all)
  const int64_t* nlist;        // device count when list != NULL
  int64_t nseq;
  const float* etab;           // [kRows][C][T][V] emission odds (chunked), full copy in global memory
  const float* tr;             // [8][T][Q] transition odds
  const float* cst;            // [kFwdConst + Q][T] D->D scan constants (forward.cu)
  int rows_smem;               // residue rows staged in shared memory (x < rows_smem)
  float* out;                  // [nseq] caller order, nats
  uint8_t* flags;              // [nseq] caller order or NULL: bit 3 set when the Forward stage ran
  unsigned long long* counter;
};

}  // namespace hmg

struct hmg_profile {
  int M = 0;
  int device = 0;
  int bias = 0, tbm = 0, tec = 0, ddbound = -32768;
  float scale_b = 0.f, scale_w = 0.f;
  std::vector<uint8_t> cost;  // [29][M]
  std::vector<int16_t> rsc;   // [29][M]
  std::vector<int16_t> tsc;   // [8][M] clamped
  bool has_tsc = false, has_ev = false;
  hmg_evparams ev{};
  int msv_fast = 0, msv_G = 0, msv_Q = 0;
  int vit_G = 0, vit_Q = 0, vit_generic = 0;
  int vit_W = 0;                    // >0: block-per-sequence kernel vit_cta_kernel<W, Q> (Q = vit_Q)
  int pair_G = 0, pair_Q = 0;       // >0: s16x2 pair kernel vit_pair_kernel<G, Q> first, the above re-scores
  bool pair_scan = false;           // pair kernel: max-plus scan Lazy-F (G = 32 only; HMG_VIT_SCAN)
  int pair_SG2 = 0;                 // >0: W = 2 without the per-row barrier, vit_cpair2_kernel<pair_Q, pair_SG2>
  int pair_wide = 0;                // one warp per sequence, Q <= 32: vit_wide_kernel<pair_Q, tm> (pair_G = 32);
                                    // 1: transitions in shared memory, 2: in tensor memory
  int pair_W = 0, pair_SG = 1;      // >0: block pair kernel vit_cpair_kernel<pair_W, pair_Q, pair_SG>
                                    //     (pair_G = 32 W; pair_SG sequences per block share its table)
  int tbm_min = 0, rmax = 0;        // pair kernel window: min_k tBM_k, max(0, max_{x,k} rsc)
  uint32_t* d_pair_rsc = nullptr;   // pair kernel tables: s16x2 emissions [kRows][G*Q] (chunk layout)
  uint32_t* d_pair_tr = nullptr;    //                     s16x2 transitions [8][G][Q]
  // device tables
  uint32_t* d_msv_prof = nullptr;   // striped s16x2 emissions
  uint8_t* d_cost = nullptr;        // [kRows][M]
  int16_t* d_rsc = nullptr;         // Viterbi emissions (layout per kernel)
  int32_t* d_tr = nullptr;          // Viterbi transitions (layout per kernel)
  size_t msv_prof_bytes = 0, vit_rsc_bytes = 0, vit_tr_bytes = 0;
  // pipeline long lane (whole-warp MSV + Viterbi), available when M <= 512
  int long_QV = 0;                  // >0: long lane available; Viterbi regs per lane (s32 nodes or pair regs)
  int long_QL = 0;                  // whole-warp MSV registers of the chunked long-lane MSV
  bool long_pair = false;           // long-lane Viterbi uses the pair lane and d_pair_* (G = 32)
  uint32_t* d_long_msv = nullptr;
  int32_t* d_long_rsc = nullptr;
  int32_t* d_long_tr = nullptr;
  // Forward stage (forward.cu): fwd_kernel<fwd_W, fwd_Q>, emission rows x < fwd_rows in shared memory
  int fwd_W = 0, fwd_Q = 0, fwd_rows = 0, fwd_S = 1;   // S sequences per block
  int fwd_T = 0;                    // threads per sequence (8 or 32 fwd_W)
  float msc_max = 0.f;              // largest emission log-odds (odds-space range check)
  float* d_fwd_e = nullptr;         // emission odds [kRows][C][T][V]
  float* d_fwd_t = nullptr;         // transition odds [8][T][Q]
  float* d_fwd_c = nullptr;         // D->D scan constants [kFwdConst + Q][T]
  // many-profile MSV (hmg_msv_batch): striped tables in other lane geometries, built on first use
  struct Tab {
    int G, Q;
    uint32_t* d;
  };
  std::vector<Tab> msv_tabs;
  // threshold tables (built on first use per F and length range, or by hmg_prepare_thresholds).
  // Every table handed out stays allocated until hmg_profile_destroy: a CUDA graph captured with
  // one, or a call still running on another stream, never sees it freed or replaced.
  std::mutex mu;
  struct Thr {
    double F = -1;
    int Lmax = -1;
    void* d = nullptr;
  };
  std::vector<Thr> thr_msv, thr_vit;
};

struct hmg_db {
  int device = 0;
  int64_t nseq = 0, residues = 0;
  int Lmax = 0;
  int64_t nwords = 0;
  std::vector<int32_t> order;      // sorted -> caller
  std::vector<int32_t> len_sorted;
  std::vector<uint32_t> woff16_h;  // host copy of the word offsets / 4 (overlapped upload parts)
  uint32_t* d_words = nullptr;
  uint32_t* d_woff16 = nullptr;
  int32_t* d_len = nullptr;
  int32_t* d_order = nullptr;     // sorted -> caller
  int32_t* d_inv = nullptr;       // caller -> sorted
  uint8_t* d_tjb = nullptr;       // [Lmax+1]
  int16_t* d_move = nullptr;      // [Lmax+1]
  std::vector<uint32_t> host_image;  // host-only handles (device < 0)
  // pipeline long lane: sequences [0, nlong) with L > long_cut, cut into chunk_rows-row chunks
  int long_cut = 0;
  int64_t nlong = 0;
  int chunk_rows = 1032;
  int64_t nchunks = 0;
  int32_t* d_chunk_start = nullptr;  // [nlong+1]
};

namespace hmg {
extern std::atomic<long long> g_launches;   // kernels launched by libhmg (hmg_kernel_launches)
// kernels / launchers (CUDA side)
cudaError_t launch_msv_fast(int G, int Q, const MsvArgs& a, cudaStream_t st, int* ok, bool pdl = false);
cudaError_t launch_msv_exact(const MsvArgs& a, int nwarps, cudaStream_t st);
cudaError_t launch_vit_reg(int G, int Q, const VitArgs& a, cudaStream_t st, int* ok);
cudaError_t launch_vit_generic(const VitArgs& a, int nwarps, cudaStream_t st);
cudaError_t launch_pipe_long_msv(int QL, const LongArgs& a, cudaStream_t st, int* ok);
cudaError_t launch_pipe_long_vit(int QV, bool pair, const LongArgs& a, int nblocks, cudaStream_t st, int* ok);
cudaError_t launch_vit_cta(int W, int Q, const VitArgs& a, cudaStream_t st, int* ok);
cudaError_t launch_vit_pair(int G, int Q, bool scan, const VitArgs& a, cudaStream_t st, int* ok);
cudaError_t launch_vit_cpair(int W, int SG, int Q, const VitArgs& a, cudaStream_t st, int* ok);
size_t vit_cpair_smem(int W, int SG, int Q);
bool vit_cpair_available(int W, int SG, int Q);
cudaError_t launch_vit_cpair2(int SG, int Q, const VitArgs& a, cudaStream_t st, int* ok);
cudaError_t launch_vit_wide(int Q, bool tm, const VitArgs& a, cudaStream_t st, int* ok);
bool vit_wide_available(int Q);
size_t vit_wide_smem(int Q, bool tm);
size_t vit_cpair2_smem(int SG, int Q);
bool vit_cpair2_available(int SG, int Q);
int vit_pair_q_max();
size_t vit_cta_smem(int W, int Q);
int long_msv_q(int M);
int msv_q_max(int G);
int msv_table_words(int G, int Q);   // MsvLayout<G, Q>::WORDS
int vit_q_max(int G);

// many-profile MSV (msv_multi.cu)
cudaError_t launch_msv_multi(int G, int Q, const MsvMultiArgs& a, cudaStream_t st, int* ok);
cudaError_t launch_msv_pairs_exact(const MsvPairArgs& a, int nwarps, cudaStream_t st);
cudaError_t select_redo_pairs(const uint8_t* raw_sorted, int64_t n, int64_t* list, int64_t* count,
                              cudaStream_t st);
cudaError_t msv_flags_multi(const uint8_t* raw_sorted, int nprof, const int32_t* len, const int32_t* order,
                            int64_t nseq, const uint16_t* const* thr, const int* rowmap, uint8_t* raw_out,
                            uint8_t* pass_out, cudaStream_t st, uint8_t* pass_sorted = nullptr);

// pipeline helpers (pipeline.cu)
cudaError_t select_redo(const uint8_t* raw_sorted, int64_t n, int32_t* list, int64_t* count, void* tmp,
                        cudaStream_t st);
cudaError_t msv_finish(const uint8_t* raw_sorted, const int32_t* len, const int32_t* order, int64_t n,
                       const uint16_t* thr, uint8_t* raw_out, uint8_t* pass_out, int32_t* surv_sorted,
                       int64_t* nsurv, int32_t* surv_caller, void* tmp, cudaStream_t st);
cudaError_t vit_finish(const int16_t* raw_sorted, const int32_t* list, const int64_t* nlist, int64_t nmax,
                       const int32_t* len, const int32_t* order, const int32_t* thr, int16_t* raw_out,
                       uint8_t* pass_out, uint8_t* flags_out, cudaStream_t st, uint8_t* pass_sorted = nullptr);
cudaError_t compact_flags(const uint8_t* flag_sorted, int64_t n, const int32_t* order, int32_t* ids_sorted,
                          int32_t* ids_caller, int64_t* count, void* tmp, cudaStream_t st);
size_t compact_rows_tmp_bytes(int64_t n, int rows);
cudaError_t compact_rows(const uint8_t* flag, int rows, int64_t n, const int32_t* order, int32_t* ids_sorted,
                         int32_t* ids_caller, int64_t* counts, const int* rowmap, void* tmp, cudaStream_t st);

// Forward stage (forward.cu)
// T = threads per sequence (8: sub-warp lane groups; 32 W: W warps)
bool fwd_geometry(int M, int* T, int* Q, int qmax);
size_t fwd_smem(int T, int Q, int rows, int S);
int fwd_pick_s(int T, int Q, int rows);
void fwd_tables(int M, int T, int Q, const float* msc, const float* tsc, std::vector<float>* etab,
                std::vector<float>* tr, std::vector<float>* cst);
cudaError_t launch_fwd(int T, int Q, int S, int rows_smem, const FwdArgs& a, cudaStream_t st, int* ok);
cudaError_t to_sorted_ids(const int32_t* caller_ids, int64_t n, const int32_t* inv_order, int32_t* sorted_ids,
                          cudaStream_t st);
cudaError_t set_count(int64_t* d, int64_t v, cudaStream_t st);
size_t scan_tmp_bytes(int64_t n);

}  // namespace hmg
