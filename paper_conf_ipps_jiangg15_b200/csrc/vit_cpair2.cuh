// vit_cpair2.cuh -- Viterbi filter (Alg 2, + Lazy-F, P:519-533 / Fig 7) for long models
// (1024 < M <= 2048): two warps per sequence, two cells per register (the s16x2 offset arithmetic
// of vit_pair.cuh, the virtual-warp layout of vit_cpair.cuh with W = 2), and NO block barrier on
// the row's critical path.
//
// vit_cpair_kernel<W,...> joins the W warps of a sequence with one full barrier per row, after
// which the cross-warp D->D carry is folded in closed form and the next row's diagonal carries are
// rebuilt -- ~140 instructions of latency-bound overhead per row beside 140 DPX ops of cell work,
// with only four sequences per SM (254 registers) to hide it (profiles/ncu_vit_cpair_r02a.md: ALU
// 62%, issue 43%).  Here each warp *publishes* its row (lane 31's M, I, D and the warp's outgoing
// D carry) and signals it with a non-blocking `bar.arrive`; the other warp waits for it with
// `bar.sync` only in the middle of its NEXT row, after the half of the row that does not need it:
//
//   phase A (row i, needs only this warp's row i-1):  I(i,k) for every node, and the partial
//            M(i,k) = max(B->M_k, M(i-1,k-1) + tMM_k, I(i-1,k-1) + tIM_k) for k > first node;
//   wait    the other warp's publication of row i-1;
//   phase B  fold the cross-warp D->D carry into D(i-1,.) (Lazy-F, reading R19; closed form for
//            W = 2), the diagonal carries into the first node, M(i,k) = max(partial, D(i-1,k-1) +
//            tDM_k) + e, the row maximum, the D chain of row i inside the warp; publish row i.
//
// Virtual warps (as vit_cpair.cuh): v0 = low halves of warp 0, v1 = low halves of warp 1, v2 = high
// halves of warp 0, v3 = high halves of warp 1.  With outgoing carries WO_v (zero carry in) and
// tDD sums BW_v, the carries into the virtual warps are c0 = 0, c1 = WO0, c2 = max(WO1, c1 + BW1),
// c3 = max(WO2, c2 + BW2) (max-plus, floored at 0 in the offset domain).
//
// Hits (a row whose maximum could move xB, or overflow; Alg 2 l.22-24, reading R17) are voted per
// warp and published with the row; both warps act on a hit of row i at the same point of row i+1
// (rebase + new B->M terms).  Row i+1's phase A ran with the old B->M terms: on the rebased
// offset map every operation commutes, and the new B->M terms only grow, so
// max(rebased partial, new Bk) is exact.  Everything else -- floor F, safe window, re-score list
// -- is vit_pair.cuh's.
//
// Registers set the sequences in flight (two warps of 64 K 32-bit registers per SM).  TSM = 0 keeps
// all seven transition vectors in registers (255 registers: 4 sequences per SM); TSM = 1 streams
// the two only the I update uses (tMI, tII) from shared memory; TSM = 2 streams
// the four that phase A uses (tMM, tIM, tMI, tII) from shared memory, one copy per block (about
// 160 registers: 6 sequences per SM at the cost of 8 more bytes of shared-memory reads per cell).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"
#include "msv.cuh"        // load_row
#include "vit_pair.cuh"   // kRedo
#include "vit_cpair.cuh"  // group_sync, group_sync_or, lo16, hi16, pack16

namespace hmg {

template <int Q, int SG, int TSM>
struct VitCP2Smem {
  static constexpr int NT = 64;
  static constexpr int ROWW = Q * NT;            // s16x2 words per residue row / per vector
  static constexpr int SROWS = 21;               // 20 canonical residues + X (code 26)
  static constexpr int TROWS = TSM ? 4 : 0;      // tMM, tIM, tMI, tII in shared memory
  static constexpr size_t table_words = (size_t)(SROWS + TROWS) * ROWW;
  static constexpr int KON = 0;                  // [4] block constants: BW1, BW2, K1, K2
  static constexpr int G0 = 4;
  // per group (u32 words, offset G0 + GRP * group)
  static constexpr int BK = 0;                   // [ROWW] B->M terms Bk' (load_row layout)
  static constexpr int XC = ROWW;                // [2 parity][2 warps] uint4: M, I, D' of lane 31, WO | hit << 31
  static constexpr int RX = XC + 16;             // [2] per-warp R maximum (hit rows, final)
  static constexpr int NX = RX + 2;              // next sequence index (long long)
  static constexpr int GRP = (NX + 2 + 3) / 4 * 4;
  static constexpr size_t bytes = sizeof(uint32_t) * (table_words + G0 + (size_t)SG * GRP);
};

__device__ __forceinline__ void bar_arrive(int id, int nthreads) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// inverse of load_row: this thread's Q words into a [chunk][lane][4] striped row
template <int G, int Q>
__device__ __forceinline__ void store_row(uint32_t* row, int z, const uint32_t (&v)[Q]) {
  using C = Chunks<Q>;
#pragma unroll
  for (int c = 0; c < C::n4; ++c)
    *reinterpret_cast<uint4*>(row + c * 4 * G + z * 4) = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  if constexpr (C::has2)
    *reinterpret_cast<uint2*>(row + C::n4 * 4 * G + z * 2) = make_uint2(v[4 * C::n4], v[4 * C::n4 + 1]);
  if constexpr (C::has1) row[(C::n4 * 4 + (C::has2 ? 2 : 0)) * G + z] = v[Q - 1];
}

// load_row from a 32-bit shared-memory address (ld.shared: no generic-to-shared conversion per row)
template <int G, int Q>
__device__ __forceinline__ void lds_row(uint32_t row_s, int z, uint32_t (&e)[Q]) {
  using C = Chunks<Q>;
#pragma unroll
  for (int c = 0; c < C::n4; ++c)
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(e[4 * c]), "=r"(e[4 * c + 1]), "=r"(e[4 * c + 2]), "=r"(e[4 * c + 3])
                 : "r"(row_s + (uint32_t)(c * 4 * G + z * 4) * 4u));
  if constexpr (C::has2)
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(e[4 * C::n4]), "=r"(e[4 * C::n4 + 1])
                 : "r"(row_s + (uint32_t)(C::n4 * 4 * G + z * 2) * 4u));
  if constexpr (C::has1)
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(e[Q - 1])
                 : "r"(row_s + (uint32_t)((C::n4 * 4 + (C::has2 ? 2 : 0)) * G + z) * 4u));
}

// s16x2 with both halves clamped below at -32768 (tDD sums: relu(c + sum) is exact with the clamp)
__device__ __forceinline__ uint32_t clamp_pack(int lo, int hi) {
  return (uint32_t)(uint16_t)max(lo, -32768) | ((uint32_t)(uint16_t)max(hi, -32768) << 16);
}

template <int Q, int SG, int TSM>
__global__ void __launch_bounds__(64 * SG, (TSM && SG == 3) ? 2 : 1) vit_cpair2_kernel(const VitArgs a) {
  static_assert(SG >= 1 && SG <= 3, "5 named barriers per sequence group, ids 1..15");
  using S = VitCP2Smem<Q, SG, TSM>;
  constexpr int NT = S::NT;
  constexpr int ROWW = S::ROWW;
  extern __shared__ uint4 smem4[];
  uint32_t* sm = reinterpret_cast<uint32_t*>(smem4);
  const uint32_t* tr = reinterpret_cast<const uint32_t*>(a.tr);
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    constexpr int R16 = ROWW / 4;
    for (int i = threadIdx.x; i < 20 * R16; i += blockDim.x) smem4[i] = src[i];
    for (int i = threadIdx.x; i < R16; i += blockDim.x) smem4[20 * R16 + i] = src[26 * R16 + i];
    if constexpr (TSM) {                         // [tMM, tIM, tMI, tII] in the load_row chunk layout
      const int vsel[4] = {1, 2, 5, 6};
      for (int i = threadIdx.x; i < 4 * ROWW; i += blockDim.x) {
        const int v = i / ROWW, o = i - v * ROWW;          // o = thread z, register q of vector v
        const int z = o / Q, q = o - z * Q;
        using C = Chunks<Q>;                     // where load_row finds word q of thread z
        int pos;
        if (q < 4 * C::n4) pos = (q >> 2) * 4 * NT + z * 4 + (q & 3);
        else if (C::has2 && q < 4 * C::n4 + 2) pos = C::n4 * 4 * NT + z * 2 + (q - 4 * C::n4);
        else pos = (C::n4 * 4 + (C::has2 ? 2 : 0)) * NT + z;
        sm[(size_t)(S::SROWS + v) * ROWW + pos] = tr[vsel[v] * NT * Q + o];
      }
    }
  }
  const uint32_t* ttab = sm + (size_t)S::SROWS * ROWW;     // TSM: tMM, tIM, tMI, tII rows
  uint32_t* scb = sm + S::table_words;
  const int grp = threadIdx.x / NT;
  uint32_t* gs = scb + S::G0 + grp * S::GRP;
  uint32_t* bks = gs + S::BK;
  uint4* xcs = reinterpret_cast<uint4*>(gs + S::XC);
  long long* s_next = reinterpret_cast<long long*>(gs + S::NX);
  const int g = threadIdx.x - grp * NT;
  const int w = g >> 5, lane = g & 31;
  const int bfull = 1 + 5 * grp;                 // both warps
  const int bmine = bfull + 1 + 2 * w;           // + parity: this warp published a row
  const int bother = bfull + 3 - 2 * w;          // + parity: the other warp published a row

  constexpr int QR = TSM == 2 ? 1 : Q;           // register copies of tMM, tIM (TSM 2: shared memory)
  constexpr int QI = TSM ? 1 : Q;                // register copies of tMI, tII (TSM 1, 2: shared memory)
  uint32_t tMM[QR], tIM[QR], tMI[QI], tII[QI];
  uint32_t tDM[Q], tMD[Q], tDD[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = g * Q + q;
    if constexpr (TSM < 2) { tMM[q] = tr[1 * NT * Q + o]; tIM[q] = tr[2 * NT * Q + o]; }
    if constexpr (TSM == 0) { tMI[q] = tr[5 * NT * Q + o]; tII[q] = tr[6 * NT * Q + o]; }
    tDM[q] = tr[3 * NT * Q + o]; tMD[q] = tr[4 * NT * Q + o]; tDD[q] = tr[7 * NT * Q + o];
  }
  // per half: sum of the thread's tDD (bs), prefix up to its last node (s31), warp-exclusive prefix (pbs)
  int bs_lo = 0, bs_hi = 0, s31_lo = 0, s31_hi = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    if (q == Q - 1) { s31_lo = bs_lo; s31_hi = bs_hi; }
    bs_lo += lo16(tDD[q]);
    bs_hi += hi16(tDD[q]);
  }
  const uint32_t bsum2 = clamp_pack(bs_lo, bs_hi);
  int pbs_lo = bs_lo, pbs_hi = bs_hi;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int yl = __shfl_up_sync(0xffffffffu, pbs_lo, o);
    const int yh = __shfl_up_sync(0xffffffffu, pbs_hi, o);
    if (lane >= o) { pbs_lo += yl; pbs_hi += yh; }
  }
  pbs_lo -= bs_lo;
  pbs_hi -= bs_hi;
  if (lane == 31 && grp == 0) {
    if (w == 1) {
      scb[S::KON + 0] = (uint32_t)(pbs_lo + bs_lo);      // BW1: tDD sum over v1
      scb[S::KON + 2] = (uint32_t)(pbs_lo + s31_lo);     // K1: v1 prefix up to its last node
    } else {
      scb[S::KON + 1] = (uint32_t)(pbs_hi + bs_hi);      // BW2: tDD sum over v2
      scb[S::KON + 3] = (uint32_t)(pbs_hi + s31_hi);     // K2: v2 prefix up to its last node
    }
  }
  __syncthreads();
  // warp-uniform constants of the closed-form carries, in s16x2 form (clamped sums: exact under relu)
  const uint32_t BW1c = clamp_pack((int)scb[S::KON + 0], 0);
  const uint32_t BW2c = clamp_pack((int)scb[S::KON + 1], 0);
  const uint32_t KD = clamp_pack(0, (int)scb[S::KON + (w ? 3 : 2)]);   // prefix to the diagonal source's last node
  const uint32_t pbs2 = clamp_pack(pbs_lo, pbs_hi);
  const uint32_t s31p = clamp_pack(s31_lo, s31_hi);
  const long long ntot = a.list ? *a.nlist : a.nseq;
  const int safe = a.safe;
  const uint32_t* rare = reinterpret_cast<const uint32_t*>(a.rsc);
  const uint32_t tab_s = (uint32_t)__cvta_generic_to_shared(sm);      // emission rows (shared window)

  for (;;) {
    if (g == 0) *s_next = (long long)atomicAdd(a.counter, 1ull);
    group_sync(bfull, NT);
    const long long idx = *s_next;
    group_sync(bfull, NT);
    if (idx >= ntot) break;
    const int s = a.list ? a.list[idx] : (int)idx;
    if (s < a.ndone && a.done[s]) continue;
    const int L = a.len[s];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    const int move = a.move[L];
    int F = max(-32768, kBaseW + move + a.tbm_min);
    int state = 0, xJ = kNegW;
    uint32_t Mc[Q], Ic[Q], Dc[Q];
    bool okv = true;
    {
      uint32_t bk[Q];
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        Mc[q] = Ic[q] = Dc[q] = 0u;                                  // Alg 2 l.9: -inf -> floor
        const uint32_t t = __ldg(tr + g * Q + q);
        const int lo = max(-32768, min(32767, kBaseW + move + lo16(t))) - F;
        const int hi = max(-32768, min(32767, kBaseW + move + hi16(t))) - F;
        okv = okv && lo <= safe && hi <= safe;
        bk[q] = pack16(max(lo, 0), max(hi, 0));
      }
      store_row<NT, Q>(bks, g, bk);
    }
    if (lane == 31) xcs[2 + w] = make_uint4(0u, 0u, 0u, 0u);        // "row -1" (parity 1)
    if (group_sync_or(bfull, NT, !okv)) state = 2;
    bar_arrive(bmine + 1, 2 * 32);
    bool pending = true;                                             // a publication not yet consumed
    uint32_t R = 0u, ci = 0u;
    int thr = min(min(kBaseW + 501, 32767) - F, safe + 1);           // in the offset domain
    uint32_t thrv = (uint32_t)(0x8000 - thr) * 0x10001u;
    int par = 0;
    // residues, one per row: 6 per packed word, the next word prefetched
    const int nw = (L + 5) / 6;
    uint32_t wv = __ldcg(wp), wnxt = nw > 1 ? __ldcg(wp + 1) : ~0u;
    int wpos = 1, sh = 0;
    auto next_x = [&]() -> int {
      if (sh == 6) {
        wv = wnxt;
        ++wpos;
        wnxt = wpos < nw ? __ldcg(wp + wpos) : ~0u;
        sh = 0;
      }
      const int xx = wv & 31;
      wv >>= 5;
      ++sh;
      return xx;
    };
    uint32_t cM = 0u, cI = 0u, mp[Q];
    // phase A of a row: this warp's previous row only -- I(i, .) and the partial M(i, .)
    auto phase_a = [&]() {
        cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1);
        cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1);
        load_row<NT, Q>(bks, g, mp);                 // Bk'
        if constexpr (TSM) {
          // the four vectors chunk by chunk (one LDS.128 of each per 4 registers), highest first
          using C = Chunks<Q>;
          uint32_t tm0 = 0u, ti0 = 0u;
#pragma unroll
          for (int c = C::n4 + (C::has2 ? 1 : 0) + (C::has1 ? 1 : 0) - 1; c >= 0; --c) {
            int q0, nq, off;
            if (c < C::n4) { q0 = 4 * c; nq = 4; off = c * 4 * NT + g * 4; }
            else if (C::has2 && c == C::n4) { q0 = 4 * C::n4; nq = 2; off = C::n4 * 4 * NT + g * 2; }
            else { q0 = Q - 1; nq = 1; off = (C::n4 * 4 + (C::has2 ? 2 : 0)) * NT + g; }
            uint32_t tmm[4], tim[4], tmi[4], tii[4];
            if (nq == 4) {
              if constexpr (TSM == 2) {
                const uint4 v0 = *reinterpret_cast<const uint4*>(ttab + 0 * ROWW + off);
                const uint4 v1 = *reinterpret_cast<const uint4*>(ttab + 1 * ROWW + off);
                tmm[0] = v0.x; tmm[1] = v0.y; tmm[2] = v0.z; tmm[3] = v0.w;
                tim[0] = v1.x; tim[1] = v1.y; tim[2] = v1.z; tim[3] = v1.w;
              }
              const uint4 v2 = *reinterpret_cast<const uint4*>(ttab + 2 * ROWW + off);
              const uint4 v3 = *reinterpret_cast<const uint4*>(ttab + 3 * ROWW + off);
              tmi[0] = v2.x; tmi[1] = v2.y; tmi[2] = v2.z; tmi[3] = v2.w;
              tii[0] = v3.x; tii[1] = v3.y; tii[2] = v3.z; tii[3] = v3.w;
            } else if (nq == 2) {
              if constexpr (TSM == 2) {
                const uint2 v0 = *reinterpret_cast<const uint2*>(ttab + 0 * ROWW + off);
                const uint2 v1 = *reinterpret_cast<const uint2*>(ttab + 1 * ROWW + off);
                tmm[0] = v0.x; tmm[1] = v0.y; tim[0] = v1.x; tim[1] = v1.y;
              }
              const uint2 v2 = *reinterpret_cast<const uint2*>(ttab + 2 * ROWW + off);
              const uint2 v3 = *reinterpret_cast<const uint2*>(ttab + 3 * ROWW + off);
              tmi[0] = v2.x; tmi[1] = v2.y; tii[0] = v3.x; tii[1] = v3.y;
            } else {
              if constexpr (TSM == 2) { tmm[0] = ttab[0 * ROWW + off]; tim[0] = ttab[1 * ROWW + off]; }
              tmi[0] = ttab[2 * ROWW + off]; tii[0] = ttab[3 * ROWW + off];
            }
            if constexpr (TSM == 1) {
#pragma unroll
              for (int jj = 0; jj < 4; ++jj)
                if (jj < nq) { tmm[jj] = tMM[q0 + jj]; tim[jj] = tIM[q0 + jj]; }
            }
#pragma unroll
            for (int j = nq - 1; j >= 0; --j) {
              const int q = q0 + j;
              if (q) {
                mp[q] = __viaddmax_s16x2(Mc[q - 1], tmm[j], mp[q]);
                mp[q] = __viaddmax_s16x2(Ic[q - 1], tim[j], mp[q]);
              } else {
                tm0 = tmm[0];
                ti0 = tim[0];
              }
              Ic[q] = __viaddmax_s16x2(Ic[q], tii[j], __viaddmax_s16x2_relu(Mc[q], tmi[j], tmi[j]));
            }
          }
          if (lane) {                                // first node's partial M from lane-1 (lane 0: below)
            mp[0] = __viaddmax_s16x2(cM, tm0, mp[0]);
            mp[0] = __viaddmax_s16x2(cI, ti0, mp[0]);
          }
          cM = tm0;                                  // lane 0 keeps tMM, tIM of its first node
          cI = ti0;
        } else {
#pragma unroll
          for (int q = Q - 1; q >= 0; --q) {
            if (q) {
              mp[q] = __viaddmax_s16x2(Mc[q - 1], tMM[q], mp[q]);
              mp[q] = __viaddmax_s16x2(Ic[q - 1], tIM[q], mp[q]);
            }
            Ic[q] = __viaddmax_s16x2(Ic[q], tII[q], __viaddmax_s16x2_relu(Mc[q], tMI[q], tMI[q]));
          }
          if (lane) {
            mp[0] = __viaddmax_s16x2(cM, tMM[0], mp[0]);
            mp[0] = __viaddmax_s16x2(cI, tIM[0], mp[0]);
          }
          cM = tMM[0];
          cI = tIM[0];
        }
    };
    // the D->D chain of row i inside the thread: partial D(i, k+1) = M(i, k) + tMD (reading R16)
    uint32_t cl = 0u;
    auto d_chain = [&]() {
      Dc[0] = 0u;
#pragma unroll
      for (int q = 1; q < Q; ++q)
        Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], __viaddmax_s16x2_relu(Mc[q - 1], tMD[q - 1], tMD[q - 1]));
      cl = __viaddmax_s16x2(Dc[Q - 1], tDD[Q - 1], __viaddmax_s16x2_relu(Mc[Q - 1], tMD[Q - 1], tMD[Q - 1]));
    };
    // (phase A of row i+1 interleaved with row i's D chain, before row i's publication, measured
    //  11% slower: it delays the publication the other warp waits for; profiles/cpair2_r02f.jsonl)
    for (int i = 0; i < L && state == 0; ++i) {
      const int x = next_x();
      phase_a();
      // ---------------- wait for the other warp's row i-1
      group_sync(bother + (par ^ 1), 2 * 32);
      pending = false;
      uint4 xm = xcs[(par ^ 1) * 2 + w];
      uint4 xo = xcs[(par ^ 1) * 2 + (w ^ 1)];
      if ((xm.w | xo.w) >> 31) {                   // Alg 2 l.22-24 on a hit row (both warps)
        uint32_t mm = R;
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 16));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 8));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 4));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 2));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 1));
        if (lane == 0) gs[S::RX + w] = mm;
        group_sync(bfull, NT);
        const uint32_t r0 = gs[S::RX], r1 = gs[S::RX + 1];
        const int mx = max(max(lo16(r0), hi16(r0)), max(lo16(r1), hi16(r1)));
        bool bad = false;
        if (mx > safe) {
          state = 2;                                   // beyond the 16-bit window: s32 re-score
        } else if (mx + F >= 32767) {
          state = 1;                                   // reading R17: overflow -> +inf, pass
        } else {
          xJ = mx + F - 500;                           // E->J (and E->C: xC == xJ)
          const int xB = max(xJ, kBaseW) + move;
          const int Fn = max(-32768, min(32767, xB + a.tbm_min));
          const int d = Fn - F;
          xm.w &= 0x7fff7fffu;
          xo.w &= 0x7fff7fffu;
          if (d > 0) {                                 // raise the floor: v' <- max(v' - d, 0)
            const uint32_t n = d >= 32768 ? 0x80008000u : (uint32_t)(uint16_t)(-d) * 0x10001u;
#pragma unroll
            for (int q = 0; q < Q; ++q) {
              Mc[q] = __viaddmax_s16x2_relu(Mc[q], n, n);
              Ic[q] = __viaddmax_s16x2_relu(Ic[q], n, n);
              Dc[q] = __viaddmax_s16x2_relu(Dc[q], n, n);
              mp[q] = __viaddmax_s16x2_relu(mp[q], n, n);
            }
            R = __viaddmax_s16x2_relu(R, n, n);
            ci = __viaddmax_s16x2_relu(ci, n, n);
            xm = make_uint4(__viaddmax_s16x2_relu(xm.x, n, n), __viaddmax_s16x2_relu(xm.y, n, n),
                            __viaddmax_s16x2_relu(xm.z, n, n), __viaddmax_s16x2_relu(xm.w, n, n));
            xo = make_uint4(__viaddmax_s16x2_relu(xo.x, n, n), __viaddmax_s16x2_relu(xo.y, n, n),
                            __viaddmax_s16x2_relu(xo.z, n, n), __viaddmax_s16x2_relu(xo.w, n, n));
          }
          F = Fn;
          uint32_t bk[Q];
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            const uint32_t t = __ldg(tr + g * Q + q);
            const int lo = max(-32768, min(32767, xB + lo16(t))) - F;
            const int hi = max(-32768, min(32767, xB + hi16(t))) - F;
            bad = bad || lo > safe || hi > safe;
            bk[q] = pack16(max(lo, 0), max(hi, 0));
            mp[q] = __vmaxs2(mp[q], bk[q]);            // new B->M terms only grow
          }
          store_row<NT, Q>(bks, g, bk);
          thr = min(min(max(xJ, kBaseW) + 501, 32767) - F, safe + 1);
          thrv = (uint32_t)(0x8000 - thr) * 0x10001u;
        }
        if (group_sync_or(bfull, NT, bad)) state = 2;
        if (state) break;
      }
      // cross-warp D->D carries (closed form for W = 2, s16x2): with A = WO of warp 0 (v0 | v2),
      // B = WO of warp 1 (v1 | v3): c1 = A.lo, c2 = max(B.lo, relu(c1 + BW1)), c3 = max(A.hi, relu(c2 + BW2))
      const uint32_t A = (w ? xo.w : xm.w) & 0x7fff7fffu, B = (w ? xm.w : xo.w) & 0x7fff7fffu;
      const uint32_t c2 = __viaddmax_s16x2_relu(A, BW1c, B) & 0xffffu;              // (c2, 0)
      const uint32_t c2h = c2 << 16;                                                   // (0, c2)
      // warp 0: (0, c2); warp 1: (c1, c3), c3 = max(A.hi, relu(c2 + BW2)) in the high half
      const uint32_t cw = w ? __viaddmax_s16x2_relu(c2h, BW2c << 16, A) : c2h;
      // incoming carry of this lane: max(intra-warp ci, relu(cw + prefix of the lanes before))
      const uint32_t cf = __viaddmax_s16x2_relu(cw, pbs2, ci);
      {                                            // D(i-1, .) += carry (Lazy-F, reading R19)
        bool imp = __vmaxs2(cf, Dc[0]) != Dc[0];
        Dc[0] = __vmaxs2(Dc[0], cf);
        constexpr int K0 = Q <= 4 ? Q : 2;
#pragma unroll
        for (int q = 1; q < K0; ++q) {
          const uint32_t nd = __viaddmax_s16x2_relu(Dc[q - 1], tDD[q - 1], tDD[q - 1]);
          imp = imp && (__vmaxs2(nd, Dc[q]) != Dc[q]);
          Dc[q] = __vmaxs2(Dc[q], nd);
        }
        if constexpr (K0 < Q) {
          if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
            for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], Dc[q]);
          }
        }
      }
      // diagonal D carry into the first node: row i-1 at the last node of the previous virtual warp
      uint32_t cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1);
      if (lane == 0) {
        // warp 1: lo <- v0 (carry 0), hi <- v2 (carry c2); warp 0: lo <- floor, hi <- v1 (carry c1)
        const uint32_t srcM = w ? xo.x : xo.x << 16, srcI = w ? xo.y : xo.y << 16;
        const uint32_t dsrc = __viaddmax_s16x2_relu(w ? c2h : A << 16, KD, w ? xo.z : xo.z << 16);
        mp[0] = __viaddmax_s16x2(srcM, cM, mp[0]);  // cM, cI hold tMM, tIM of the first node
        mp[0] = __viaddmax_s16x2(srcI, cI, mp[0]);
        cD = dsrc;
      }
      // ---------------- phase B: M(i, .) (Alg 2 l.16 + emission, reading R15), row max, D chain
      {
        uint32_t e[Q];
        if (x < 20 || x == 26) {                  // shared memory
          lds_row<NT, Q>(tab_s + (uint32_t)((x < 20 ? x : 20) * ROWW) * 4u, g, e);
        } else {                                   // rare codes (B J Z O U, gaps): L2
          load_row<NT, Q>(rare + x * ROWW, g, e);
        }
#pragma unroll
        for (int q = Q - 1; q >= 0; --q) {
          const uint32_t m = __viaddmax_s16x2(q ? Dc[q - 1] : cD, tDM[q], mp[q]);
          Mc[q] = __viaddmax_s16x2_relu(m, e[q], e[q]);
        }
      }
      // row maximum: a max3 / max tree (depth 3) instead of a Q/2-long VIMNMX3 chain through R
      {
        constexpr int G3 = Q / 3, N0 = G3 + (Q % 3 ? 1 : 0), N1 = (N0 + 1) / 2;
        uint32_t t[N0];
#pragma unroll
        for (int k = 0; k < G3; ++k) t[k] = __vimax3_s16x2(Mc[3 * k], Mc[3 * k + 1], Mc[3 * k + 2]);
        if constexpr (Q % 3 == 2) t[G3] = __vmaxs2(Mc[Q - 2], Mc[Q - 1]);
        if constexpr (Q % 3 == 1) t[G3] = Mc[Q - 1];
        uint32_t u[N1];
#pragma unroll
        for (int k = 0; k < N1; ++k) u[k] = (2 * k + 1 < N0) ? __vmaxs2(t[2 * k], t[2 * k + 1]) : t[2 * k];
#pragma unroll
        for (int k = 0; k < N1; ++k) R = __vmaxs2(R, u[k]);
      }
      const uint32_t mlast = Mc[Q - 1], ilast = Ic[Q - 1];   // row i at the last node (publication)
      d_chain();
      // carries inside the warp: ci = outgoing of lane-1 (lane 0: floor), until no lane changes
      uint32_t out = cl;
      for (;;) {
        ci = __shfl_up_sync(0xffffffffu, out, 1);
        if (lane == 0) ci = 0u;
        const uint32_t o2 = __viaddmax_s16x2_relu(ci, bsum2, cl);    // max(cl, relu(ci + bsum))
        const bool chg = o2 != out;
        out = o2;
        if (!__any_sync(0xffffffffu, chg)) break;
      }
      const bool hit = __any_sync(0xffffffffu, (__vadd2(R, thrv) & 0x80008000u) != 0u);
      if (lane == 31)
        xcs[par * 2 + w] = make_uint4(mlast, ilast, __viaddmax_s16x2_relu(ci, s31p, Dc[Q - 1]),
                                      out | (hit ? 0x80000000u : 0u));
      bar_arrive(bmine + par, 2 * 32);
      pending = true;
      par ^= 1;
    }
    if (pending) group_sync(bother + (par ^ 1), 2 * 32);   // consume the other warp's last row
    // the last row's hit (if any) and xC = max over rows of xE - 500
    uint32_t mm = R;
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 16));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 8));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 4));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 2));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 1));
    if (lane == 0) gs[S::RX + w] = mm;
    group_sync(bfull, NT);
    if (g == 0) {
      const uint32_t r0 = gs[S::RX], r1 = gs[S::RX + 1];
      const int mx = max(max(lo16(r0), hi16(r0)), max(lo16(r1), hi16(r1)));
      int raw;
      if (state == 1) raw = 32767;
      else if (state == 2 || mx > safe) raw = kRedo;
      else if (mx + F >= 32767) raw = 32767;           // reading R17: overflow on the last row
      else if (mx > 0) raw = max(xJ, max(kNegW, mx + F - 500));
      else raw = xJ > kNegW ? xJ : kRedo;
      if (raw >= -32768) {
        a.raw_sorted[s] = (int16_t)raw;
      } else {
        const unsigned long long k = atomicAdd(a.redo_count, 1ull);
        a.redo_list[k] = s;
      }
    }
    group_sync(bfull, NT);
  }
}

}  // namespace hmg
