// msv.cuh -- MSV filter kernels for sm_100a (Alg 1).
//
// Fast kernel (msv_fast_kernel<G, Q>): a group of G lanes scores one sequence
// (the paper's "warp = one sequence", generalised to G in
// {4, 8, 16, 32}); 32/G sequences of equal length rank share a warp.  Each lane
// holds Q 32-bit registers of DP cells as s16x2 pairs (HMMER's Farrar striping,
// ref [19], over 2G virtual lanes: register q of lane z holds nodes z*Q+q+1 (low
// half) and (z+G)*Q+q+1 (high half)), so the diagonal dependence of Alg 1 l.15
// is register q-1 -> q inside a lane and one __shfl_sync per row across lanes
// (the paper's double buffering, becomes register renaming).
//
// Cell update: the state of a cell is
//     t_i[k] = max(s_{i-1}[k-1] + bias, B')        with B' = min(xB - tbm + bias, 255)
// and one row is a single DPX instruction per register,
//     t_{i+1}[k+1] = VIADDMNMX.S16x2(t_i[k], e[x_i][k], B')    e = bias - cost,
// which reproduces Alg 1 l.15 (max, +bias, -cost, all u8-saturating) exactly
// while no row has overflowed (proof in DESIGN.md; the u8 floor at 0 is
// absorbed by B' >= bias).  xE (Alg 1 l.16/l.20) is tracked as a running
// per-lane max R (VIMNMX3, half an instruction per register) and a per-row
// __ballot_sync against the threshold at which J->B or overflow could change;
// B' is speculated unchanged and corrected (monotone max) on the rare rows
// where the vote fires.  Valid iff bias < 66 + tbm (host check); otherwise the
// exact kernel runs.
#pragma once
#include <type_traits>
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"

namespace hmg {

// The striped table row layout for (G, Q): chunks of 4, then 2, then 1 words per
// lane; chunk c occupies G*w_c consecutive words, lane z at offset z*w_c.
template <int Q>
struct Chunks {
  static constexpr int n4 = Q / 4;
  static constexpr int r = Q % 4;
  static constexpr bool has2 = r >= 2;
  static constexpr bool has1 = (r % 2) == 1;
};

// Shared-memory layout of the striped table for lane groups of G.  For G < 8 two or more
// groups share a quarter-warp's LDS.128 wavefront while reading different residue rows; they
// get their own copy of the table, shifted by 16*G bytes inside the 128-byte bank period
// (row stride a multiple of 128 B), so their 16*G-byte chunks never share a bank.
// For G = 8 / 16 the 4-word chunks are one quarter-warp's 128 B and never conflict, but the
// remainder chunks (2 words per lane: LDS.64, split per half-warp; 1 word: LDS.32, whole warp)
// are read by 2 or 4 groups of different residue rows in one wavefront: each row holds
// 32 / (G * w) copies of such a chunk, copy j at bank offset j * G * w, and group grp reads copy
// grp % NC -- conflict-free with the row stride a multiple of 32 words (it was 3.8% of the
// config-3 kernel's shared-memory wavefronts, profiles/ncu_full_r02n.md).
// With BYTE (G = 8 / 16 and a 2-word remainder) that chunk is one word per lane holding its two
// registers as four int8 emissions (clamped at -128, exact under msv_byte_exact), in 32 / G
// per-group copies: one conflict-free LDS.32 wavefront per warp instead of the LDS.64's two, for
// two PRMT per lane-row on the ALU pipe, which has room (the kernel is bound by the shared-memory
// wavefronts: L1 99.7% busy, ALU 78%, profiles/ncu_full_r02zk.md).  Also taking the last 4-register
// chunk as int8 (one LDS.64) cut the wavefronts another 7.6% but moved the kernel onto the ALU pipe
// (89%) and measured slower (config 3 5.77 -> 5.99 ms, config 2 2.88 -> 3.44; cmp_r02zzc.jsonl).
template <int G, int Q>
struct MsvLayout {
  using C = Chunks<Q>;
  static constexpr bool BYTE = kMsvByte && (G == 8 || G == 16) && C::has2;
  static constexpr int NCB = 32 / G;                                            // copies of the byte chunk
  static constexpr int NCOPY = G < 8 ? 8 / G : 1;
  static constexpr int NC2 = G == 8 ? 2 : 1;                                    // copies of the 2-word chunk
  static constexpr int NC1 = G == 8 ? 4 : (G == 16 ? 2 : 1);                    // copies of the 1-word chunk
  static constexpr int B2 = C::n4 * 4 * G;                                      // 2-word chunk (copy 0)
  static constexpr int B1 = B2 + (C::has2 ? 2 * G * NC2 : 0);                   // 1-word chunk (copy 0)
  static constexpr int ROWW = B1 + (C::has1 ? G * NC1 : 0);
  static constexpr int STRIDE = NCOPY > 1 ? (ROWW + 31) / 32 * 32 : ROWW;       // words per row
  static constexpr int COPY = kRows * STRIDE;                                   // words per copy
  static constexpr int WORDS = ((NCOPY * COPY + (NCOPY - 1) * 4 * G) + 3) / 4 * 4;
  __host__ __device__ static constexpr int base(int grp) { return (grp % NCOPY) * (COPY + 4 * G); }
};

template <int G, int Q>
__device__ __forceinline__ void load_row(const uint32_t* __restrict__ row, int z, uint32_t (&e)[Q]) {
  using C = Chunks<Q>;
#pragma unroll
  for (int c = 0; c < C::n4; ++c) {
    uint4 v = *reinterpret_cast<const uint4*>(row + c * 4 * G + z * 4);
    e[4 * c + 0] = v.x;
    e[4 * c + 1] = v.y;
    e[4 * c + 2] = v.z;
    e[4 * c + 3] = v.w;
  }
  if constexpr (C::has2) {
    uint2 v = *reinterpret_cast<const uint2*>(row + C::n4 * 4 * G + z * 2);
    e[4 * C::n4 + 0] = v.x;
    e[4 * C::n4 + 1] = v.y;
  }
  if constexpr (C::has1) {
    e[Q - 1] = row[(C::n4 * 4 + (C::has2 ? 2 : 0)) * G + z];
  }
}

// PRMT in its default mode: a selector nibble with its top bit set replicates the sign of the byte
// it names (__byte_perm uses only the low three bits of each nibble)
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt_sext(uint32_t v) {
  uint32_t r;
  asm("prmt.b32 %0, %1, 0, %2;" : "=r"(r) : "r"(v), "n"(SEL));
  return r;
}

// load_row in the MSV layout (MsvLayout<G, Q>: remainder chunks in per-group copies)
template <int G, int Q>
__device__ __forceinline__ void load_row_msv(const uint32_t* __restrict__ row, int z, int grp, uint32_t (&e)[Q]) {
  using C = Chunks<Q>;
  using Lt = MsvLayout<G, Q>;
#pragma unroll
  for (int c = 0; c < C::n4; ++c) {
    uint4 v = *reinterpret_cast<const uint4*>(row + c * 4 * G + z * 4);
    e[4 * c + 0] = v.x;
    e[4 * c + 1] = v.y;
    e[4 * c + 2] = v.z;
    e[4 * c + 3] = v.w;
  }
  if constexpr (Lt::BYTE) {
    const uint32_t v = row[Lt::B2 + (grp % Lt::NCB) * G + z];
    e[4 * C::n4 + 0] = prmt_sext<0x9180u>(v);    // s16x2 (sext b0, sext b1)
    e[4 * C::n4 + 1] = prmt_sext<0xB3A2u>(v);    // s16x2 (sext b2, sext b3)
  } else if constexpr (C::has2) {
    uint2 v = *reinterpret_cast<const uint2*>(row + Lt::B2 + (grp % Lt::NC2) * 2 * G + z * 2);
    e[4 * C::n4 + 0] = v.x;
    e[4 * C::n4 + 1] = v.y;
  }
  if constexpr (C::has1) {
    e[Q - 1] = row[Lt::B1 + (grp % Lt::NC1) * G + z];
  }
}

// Residue stream of one sequence: 16-byte quads of packed words (24 residues) fetched two
// quads ahead, so the DRAM/L2 latency of the residue stream hides behind >= 24 DP rows even
// for short models.  Words past the sequence are all-31 (pad rows).
// (L2-only loads, not the read-only path: under hmg_pipeline_upload the image lands while the MSV
//  kernel runs, and a line shared with an earlier part may already sit in L1)
struct ResStream {
  const uint4* p;
  int nq;
  uint4 cur, nxt;
  __device__ __forceinline__ static uint4 pad() { return make_uint4(~0u, ~0u, ~0u, ~0u); }
  __device__ __forceinline__ void init(const uint32_t* wp, int nw) {
    p = reinterpret_cast<const uint4*>(wp);
    nq = (nw + 3) / 4;
    cur = nq > 0 ? __ldcg(p) : pad();
    nxt = nq > 1 ? __ldcg(p + 1) : pad();
  }
  __device__ __forceinline__ uint4 next(int iq) {   // quad iq, prefetching iq + 2
    const uint4 r = cur;
    cur = nxt;
    nxt = (iq + 2 < nq) ? __ldcg(p + iq + 2) : pad();
    return r;
  }
};

// Short rows (Q <= 8): vote once per 6-row word and replay the word on a crossing, instead of the
// branch-free pass + checked re-run of the whole batch.  Whole-warp batches (G = 32: the long
// sequences of hmg_msv's long queue and the long lane's sequential fallback) always do: a re-run
// doubles the latency of a sequence that sets the kernel's tail (config 2: 3.10 -> 2.84 ms,
// profiles/cmp_r02zl.jsonl); the long lane's sequential fallback (long.cu) runs only the checked
// pass (CHECKED below).
// MSV_WORD_VOTE_ALL builds use it for every Q <= 8 geometry (measured equal, cmp_r02zm.jsonl).
template <int G, int Q>
constexpr bool msv_word_vote() {
#ifdef MSV_WORD_VOTE_ALL
  return Q <= 8;
#else
  return G == 32 && Q <= 8;
#endif
}

__device__ __forceinline__ int msv_thr(int xJ, int bias) {
  // smallest t-scale value at which xJ could change J->B (xJ >= 190) or overflow
  int T = max(xJ, 189) + 4;
  T = min(T, 255 - bias);
  return T + bias;
}

// Score one batch of 32/G sequences (sorted indices s0 + group) with G lanes per
// sequence and Q s16x2 registers per lane, profile table `sm` in shared memory.
// CHECKED: the caller knows a cell reaches the threshold (the long lane's sequential fallback after
// a chunk crossed it): only the pass with the per-row update (no branch-free pass first)
template <int G, int Q, bool WV = msv_word_vote<G, Q>(), bool CHECKED = false>
__device__ __forceinline__ int msv_batch(const MsvArgs& a, const uint32_t* __restrict__ sm, long long s0,
                                         long long send) {
  // sm: the table as laid out by MsvLayout<G, Q>
  constexpr int ROWW = MsvLayout<G, Q>::STRIDE;    // words per residue row
  const int lane = threadIdx.x & 31;
  const int z = lane & (G - 1);
  const int grp = lane / G;
  sm += MsvLayout<G, Q>::base(grp);
  const unsigned gbits = (G == 32 ? 0xffffffffu : ((1u << G) - 1u)) << (grp * G);
  const uint32_t sel = (z == 0) ? 0x1054u : 0x3210u;   // carry fix-up for virtual lane 0 / G
  const uint32_t negpair = (uint32_t)(uint16_t)kNegE;  // low half = -inf
  const int bias = a.bias, tbm = a.tbm;

  const long long s = s0 + grp;
  const bool valid = s < send;
  const int L = valid ? a.len[s] : 0;
  int Lmax = L;                                         // sorted descending: group 0 is the longest
  if constexpr (G < 32) Lmax = __shfl_sync(0xffffffffu, L, 0);
  const uint32_t* wp = a.words + (valid ? (size_t)a.woff16[s] * 4 : 0);
  const int nw = (L + 5) / 6;
  const int tjb = valid ? a.tjb[L] : 0;

  int xJ;
  bool ovf;
  int Bp;
  uint32_t B2, thrv, R;
  uint32_t t[Q];
  auto reset = [&]() {
    xJ = 0;
    ovf = false;
    Bp = min(max(kBaseB - tjb - tbm, 0) + bias, 255);
    B2 = (uint32_t)Bp * 0x10001u;
    thrv = valid ? (uint32_t)(0x8000 - msv_thr(xJ, bias)) * 0x10001u : 0u;   // 0: never fires
#pragma unroll
    for (int q = 0; q < Q; ++q) t[q] = B2;   // row 1: max(0 + bias, B') = B'
    R = B2;
  };

  const int nqmax = (Lmax + 23) / 24;
  const int nwmax = (Lmax + 5) / 6;                     // rows stop at the group's last word
  // All rows of the batch.  CHECK: the per-row J->B / overflow vote and update (Alg 1 l.16-20)
  // after every row; without it (the first pass) the rows run branch-free.
  auto run = [&](auto check_tag) {
   constexpr bool CHECK = decltype(check_tag)::value;
   ResStream rs;
   rs.init(wp, nw);
   for (int iq = 0; iq < nqmax; ++iq) {
   uint4 w4 = rs.next(iq);
#pragma unroll 1
   for (int k = 0; k < 4; ++k) {
    if (iq * 4 + k >= nwmax) break;                     // warp-uniform (Lmax is lane 0's)
    const uint32_t w = w4.x;
    w4.x = w4.y;
    w4.y = w4.z;
    w4.z = w4.w;
    // one DP row (Alg 1 l.11-20); `check`: per-row J->B / overflow vote
    auto row = [&](int x, bool check) {
      uint32_t e[Q];
      load_row_msv<G, Q>(sm + x * ROWW, z, grp, e);
      // diagonal carry from the previous virtual lane (value after its emission)
      const uint32_t co = __vadd2(t[Q - 1], e[Q - 1]);
      uint32_t c = __shfl_sync(0xffffffffu, co, (z + G - 1) & (G - 1), G);
      c = __byte_perm(c, negpair, sel);
#pragma unroll
      for (int q = Q - 1; q >= 1; --q) t[q] = __viaddmax_s16x2(t[q - 1], e[q - 1], B2);
      t[0] = __vmaxs2(c, B2);
      // R also takes the outgoing carry co (this row's cells, the next lane's t[0] before the floor):
      // the high half of lane G-1 is node M's cell when 2GQ = M, which no lane receives
#pragma unroll
      for (int q = 0; q + 1 < Q; q += 2) R = __vimax3_s16x2(R, t[q], t[q + 1]);
      if constexpr (Q % 2) R = __vimax3_s16x2(R, t[Q - 1], co);
      else R = __vmaxs2(R, co);
      if (!check) return;
      // does any cell of this row reach the J->B / overflow threshold?
      const bool hit = (__vadd2(R, thrv) & 0x80008000u) != 0u;
      const unsigned bal = __ballot_sync(0xffffffffu, hit);
      if (bal) {
        uint32_t m = R;
#pragma unroll
        for (int o = G / 2; o >= 1; o >>= 1) m = __vmaxs2(m, __shfl_xor_sync(0xffffffffu, m, o));
        const int Rmax = max((int)(m & 0xffffu), (int)(m >> 16));
        if ((bal & gbits) && !ovf) {
          if (Rmax >= 255) {           // xE >= 255 - bias: overflow (reading R13)
            ovf = true;
            thrv = 0;
          } else {
            xJ = max(xJ, Rmax - bias - 3);                 // E->J, Alg 1 l.20
            const int xB = max(kBaseB, xJ) - tjb;          // J->B
            Bp = min(max(xB - tbm, 0) + bias, 255);
            B2 = (uint32_t)Bp * 0x10001u;
#pragma unroll
            for (int q = 0; q < Q; ++q) t[q] = __vmaxs2(t[q], B2);
            thrv = (uint32_t)(0x8000 - msv_thr(xJ, bias)) * 0x10001u;
          }
        }
      }
    };
    if constexpr (WV) {
      // short rows: vote once per word (6 rows).  R is a running max, so a threshold crossing
      // anywhere in the word shows at its end; then the word is replayed from a snapshot
      // with the per-row vote (exact, and rare: only hits).
      uint32_t ts[Q];
#pragma unroll
      for (int q = 0; q < Q; ++q) ts[q] = t[q];
      const uint32_t Rs = R;
#pragma unroll
      for (int j = 0; j < 6; ++j) row((w >> (5 * j)) & 31, false);
      if (__any_sync(0xffffffffu, (__vadd2(R, thrv) & 0x80008000u) != 0u)) {
#pragma unroll
        for (int q = 0; q < Q; ++q) t[q] = ts[q];
        R = Rs;
#pragma unroll
        for (int j = 0; j < 6; ++j) row((w >> (5 * j)) & 31, true);
      }
    } else {
#pragma unroll
      for (int j = 0; j < 6; ++j) row((w >> (5 * j)) & 31, CHECK);
    }
   }
   }
  };
  reset();
  if constexpr (WV || CHECKED) {
    run(std::true_type{});
  } else {
    // First the whole batch without the per-row update -- a branch per row pins t[] to fixed
    // registers, and ptxas then copies all Q of them back after every row (26 IMAD.MOV per row
    // at Q = 26, a third of the kernel's instructions; 9.6% of the kernel's time,
    // profiles/stage_nocheck_r02zh.jsonl); for short rows the per-word vote and its register
    // snapshot cost registers (74 at G = 16, Q = 4: three blocks per SM).  With the threshold
    // fixed and R a running max, that pass is exact unless some cell reached the J->B /
    // overflow threshold; then (rare: about 0.2% of config-3 sequences) the batch is scored
    // again with the per-row update.
    run(std::false_type{});
    if (__any_sync(0xffffffffu, (__vadd2(R, thrv) & 0x80008000u) != 0u)) {
      reset();
      run(std::true_type{});
    }
  }
  // final xJ = max over all cells of (s - 3); R holds max over t = max(s + bias, B')
  uint32_t m = R;
#pragma unroll
  for (int o = G / 2; o >= 1; o >>= 1) m = __vmaxs2(m, __shfl_xor_sync(0xffffffffu, m, o));
  const int Rmax = max((int)(m & 0xffffu), (int)(m >> 16));
  int raw;
  if (ovf) raw = 255;
  else if (Rmax > Bp) raw = max(xJ, max(Rmax - bias - 3, 0));
  else raw = 254;                   // every cell <= B': exact kernel recomputes (rare)
  if (valid && z == 0) a.raw[s] = (uint8_t)raw;
  return raw;                       // identical on the G lanes of the group
}

// Rows [r0, r1) of one sequence with a whole warp, starting from the empty state (t = B')
// `warm` rows earlier.  Exact for rows >= r0 whenever warm >= M - 1 and xB stays at its initial
// value: an MSV path is one ungapped diagonal segment per domain, so a cell of row i only
// depends on rows > i - M.  Returns false if a counted row reached the J->B /
// overflow threshold (xB would change: the caller falls back to the sequential DP);
// otherwise *rmax = max t over the counted rows.
template <int Q>
__device__ __forceinline__ bool msv_chunk(const MsvArgs& a, const uint32_t* __restrict__ sm, long long s, int r0,
                                          int r1, int warm, int* rmax) {
  constexpr int G = 32;
  constexpr int ROWW = Q * G;
  const int z = threadIdx.x & 31;
  const uint32_t sel = (z == 0) ? 0x1054u : 0x3210u;
  const uint32_t negpair = (uint32_t)(uint16_t)kNegE;
  const int bias = a.bias, tbm = a.tbm;
  const int L = a.len[s];
  const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
  const int nw = (L + 5) / 6;
  const int tjb = a.tjb[L];
  const int Bp = min(max(kBaseB - tjb - tbm, 0) + bias, 255);
  const uint32_t B2 = (uint32_t)Bp * 0x10001u;
  const uint32_t thrv = (uint32_t)(0x8000 - msv_thr(0, bias)) * 0x10001u;
  uint32_t t[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) t[q] = B2;
  uint32_t R = B2;
  const int wc = r0 / 6;                       // first counted word (r0 is a multiple of 6)
  const int wb = max(0, r0 - warm) / 6;        // first warm-up word
  const int we = min(nw, (r1 + 5) / 6);
  for (int blk = wb; blk < we; ++blk) {
    const uint32_t w = __ldcg(wp + blk);
    const bool counting = blk >= wc;
#pragma unroll
    for (int j = 0; j < 6; ++j) {
      const int x = (w >> (5 * j)) & 31;
      uint32_t e[Q];
      load_row_msv<G, Q>(sm + x * ROWW, z, 0, e);
      const uint32_t co = __vadd2(t[Q - 1], e[Q - 1]);
      uint32_t c = __shfl_sync(0xffffffffu, co, (z + G - 1) & (G - 1), G);
      c = __byte_perm(c, negpair, sel);
#pragma unroll
      for (int q = Q - 1; q >= 1; --q) t[q] = __viaddmax_s16x2(t[q - 1], e[q - 1], B2);
      t[0] = __vmaxs2(c, B2);
      if (counting) {
#pragma unroll
        for (int q = 0; q + 1 < Q; q += 2) R = __vimax3_s16x2(R, t[q], t[q + 1]);
        if constexpr (Q % 2) R = __vimax3_s16x2(R, t[Q - 1], co);     // co: as in msv_batch
        else R = __vmaxs2(R, co);
        if (__any_sync(0xffffffffu, (__vadd2(R, thrv) & 0x80008000u) != 0u)) return false;
      }
    }
  }
  uint32_t m = R;
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) m = __vmaxs2(m, __shfl_xor_sync(0xffffffffu, m, o));
  *rmax = max((int)(m & 0xffffu), (int)(m >> 16));
  return true;
}

// Long sequences (the first a.nlong in length order) use a whole warp (G = 32,
// QL registers) so their row latency stays well below the kernel's duration;
// the rest use G lanes.  Two work queues, long first.
template <int G, int Q>
struct MsvLong {
  static constexpr int QL = (G == 32) ? 0 : (G * Q + 31) / 32;
};

// Minimum resident blocks per SM for a lane geometry: forcing 3 (<= 85 registers) lets a third
// 256-thread block share the SM where the measured sweep gains (profiles/msv_minb_r01.jsonl:
// G = 8, Q = 26: -7%; G = 16, Q = 16: -15%; G = 32, Q = 24 at 2 blocks: -6%; a fourth block at
// G = 8, Q = 26 spills in the row loop: +31%); 0 = no bound.
template <int G, int Q>
constexpr int msv_min_blocks() {
  if (G == 4 && Q >= 8 && Q <= 10) return 3;
  if (G == 8 && Q >= 24) return 3;
  if (G == 16 && Q >= 14 && Q <= 18) return 3;
  if (G == 32 && Q >= 22 && Q <= 26) return 2;
  return 0;
}

template <int G, int Q>
__device__ __forceinline__ void msv_fast_body(const MsvArgs& a) {
  extern __shared__ uint4 smem4[];
  constexpr int QL = MsvLong<G, Q>::QL;
  constexpr int W0 = MsvLayout<G, Q>::WORDS;   // words of the main table (all copies)
  constexpr int W1 = kRows * QL * 32;      // words of the long-sequence table
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.prof);
    for (int i = threadIdx.x; i < (W0 + W1) / 4; i += blockDim.x) smem4[i] = src[i];
  }
  __syncthreads();
  const uint32_t* sm = reinterpret_cast<const uint32_t*>(smem4);
  const int lane = threadIdx.x & 31;
  if constexpr (QL > 0) {
    for (;;) {
      if (a.skip_long) break;
      unsigned long long b = 0;
      if (lane == 0) b = atomicAdd(a.counter + 1, 1ull);
      b = __shfl_sync(0xffffffffu, b, 0);
      if ((long long)b >= a.nlong) break;
      msv_batch<32, QL>(a, sm + W0, (long long)b, a.nlong);
    }
  }
  constexpr int NG = 32 / G;
  const long long first = (QL > 0 || a.skip_long) ? a.nlong : 0;
  // (claiming the next batch before scoring the current one measured no difference,
  //  profiles/cmp_r02zl.jsonl)
  for (;;) {
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(a.counter, (unsigned long long)NG);
    b = __shfl_sync(0xffffffffu, b, 0);
    if (first + (long long)b >= a.nseq) break;
    msv_batch<G, Q>(a, sm, first + (long long)b, a.nseq);
  }
}

template <int G, int Q>
__global__ void __launch_bounds__(256) msv_fast_kernel(const MsvArgs a) { msv_fast_body<G, Q>(a); }

template <int G, int Q, int MB>
__global__ void __launch_bounds__(256, MB) msv_fast_kernel_mb(const MsvArgs a) { msv_fast_body<G, Q>(a); }

// the kernel instantiated for (G, Q): with a minimum-blocks bound where it measured faster
template <int G, int Q>
const void* msv_fast_entry() {
  constexpr int MB = msv_min_blocks<G, Q>();
  if constexpr (MB > 0) return reinterpret_cast<const void*>(&msv_fast_kernel_mb<G, Q, MB>);
  else return reinterpret_cast<const void*>(&msv_fast_kernel<G, Q>);
}

}  // namespace hmg
