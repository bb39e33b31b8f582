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
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"
#include "msv.cuh"        // load_row
#include "vit_pair.cuh"   // kRedo
#include "vit_cpair.cuh"  // group_sync, group_sync_or, lo16, hi16, pack16

namespace hmg {

template <int Q, int SG>
struct VitCP2Smem {
  static constexpr int NT = 64;
  static constexpr int ROWW = Q * NT;            // s16x2 words per residue row
  static constexpr int SROWS = 21;               // 20 canonical residues + X (code 26)
  static constexpr size_t table_bytes = (size_t)SROWS * ROWW * 4;
  static constexpr int KON = 0;                  // [4] block constants: BW1, BW2, K1, K2
  static constexpr int G0 = 4;
  // per group (u32 words, offset G0 + GRP * group)
  static constexpr int BK = 0;                   // [ROWW] B->M terms Bk' (load_row layout)
  static constexpr int XC = ROWW;                // [2 parity][2 warps] uint4: M, I, D' of lane 31, WO | hit << 31
  static constexpr int RX = XC + 16;             // [2] per-warp R maximum (hit rows, final)
  static constexpr int NX = RX + 2;              // next sequence index (long long)
  static constexpr int GRP = (NX + 2 + 3) / 4 * 4;
  static constexpr size_t bytes = table_bytes + sizeof(uint32_t) * (G0 + (size_t)SG * GRP);
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

__device__ __forceinline__ uint32_t relu_pack(int lo, int hi) {   // clamp both to [0, 32767], pack
  return pack16(min(32767, max(0, lo)), min(32767, max(0, hi)));
}

template <int Q, int SG>
__global__ void __launch_bounds__(64 * SG, 1) vit_cpair2_kernel(const VitArgs a) {
  static_assert(SG >= 1 && SG <= 3, "5 named barriers per sequence group, ids 1..15");
  using S = VitCP2Smem<Q, SG>;
  constexpr int NT = S::NT;
  constexpr int ROWW = S::ROWW;
  extern __shared__ uint4 smem4[];
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    constexpr int R16 = ROWW / 4;
    for (int i = threadIdx.x; i < 20 * R16; i += blockDim.x) smem4[i] = src[i];
    for (int i = threadIdx.x; i < R16; i += blockDim.x) smem4[20 * R16 + i] = src[26 * R16 + i];
  }
  const uint32_t* tab = reinterpret_cast<const uint32_t*>(smem4);
  uint32_t* scb = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(smem4) + S::table_bytes);
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
  const uint32_t* tr = reinterpret_cast<const uint32_t*>(a.tr);

  uint32_t tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = g * Q + q;
    tMM[q] = tr[1 * NT * Q + o]; tIM[q] = tr[2 * NT * Q + o]; tDM[q] = tr[3 * NT * Q + o];
    tMD[q] = tr[4 * NT * Q + o]; tMI[q] = tr[5 * NT * Q + o]; tII[q] = tr[6 * NT * Q + o];
    tDD[q] = tr[7 * NT * Q + o];
  }
  // per half: sum of the thread's tDD (bs), prefix up to its last node (s31), warp-exclusive prefix (pbs)
  int bs_lo = 0, bs_hi = 0, s31_lo = 0, s31_hi = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    if (q == Q - 1) { s31_lo = bs_lo; s31_hi = bs_hi; }
    bs_lo += lo16(tDD[q]);
    bs_hi += hi16(tDD[q]);
  }
  const uint32_t bsum2 = (uint32_t)(uint16_t)max(bs_lo, -32768) | ((uint32_t)(uint16_t)max(bs_hi, -32768) << 16);
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
  const int BW1 = (int)scb[S::KON + 0], BW2 = (int)scb[S::KON + 1];
  const int K1 = (int)scb[S::KON + 2], K2 = (int)scb[S::KON + 3];
  const uint32_t s31p = (uint32_t)(uint16_t)max(s31_lo, -32768) | ((uint32_t)(uint16_t)max(s31_hi, -32768) << 16);
  const long long ntot = a.list ? *a.nlist : a.nseq;
  const int safe = a.safe;

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
    int par = 0;
    const int nw = (L + 5) / 6;
    uint32_t wnxt = __ldcg(wp);
    for (int iw = 0; iw < nw && state == 0; ++iw) {
     uint32_t wv = wnxt;
     wnxt = iw + 1 < nw ? __ldcg(wp + iw + 1) : ~0u;
#pragma unroll 1
     for (int j = 0; j < 6; ++j) {
      const int x = wv & 31;                       // block-uniform: uniform branches below
      wv >>= 5;
      if (x == 31) break;                          // pad slots of the last word
      // ---------------- phase A: this warp's row i-1 only
      uint32_t cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1);
      uint32_t cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1);
      uint32_t mp[Q];
      load_row<NT, Q>(bks, g, mp);                 // Bk'
#pragma unroll
      for (int q = Q - 1; q >= 1; --q) {
        mp[q] = __viaddmax_s16x2(Mc[q - 1], tMM[q], mp[q]);
        mp[q] = __viaddmax_s16x2(Ic[q - 1], tIM[q], mp[q]);
      }
#pragma unroll
      for (int q = 0; q < Q; ++q) Ic[q] = __viaddmax_s16x2(Ic[q], tII[q], __viaddmax_s16x2_relu(Mc[q], tMI[q], tMI[q]));
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
            cM = __viaddmax_s16x2_relu(cM, n, n);
            cI = __viaddmax_s16x2_relu(cI, n, n);
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
        }
        if (group_sync_or(bfull, NT, bad)) state = 2;
        if (state) break;
      }
      // cross-warp D->D carries into v0..v3 (closed form for W = 2), this warp's halves
      const uint32_t wo0 = (w ? xo.w : xm.w) & 0x7fff7fffu, wo1 = (w ? xm.w : xo.w) & 0x7fff7fffu;
      const int c1 = lo16(wo0);
      const int c2 = max(lo16(wo1), max(0, c1 + BW1));
      const int cw_lo = w ? c1 : 0;
      const int cw_hi = w ? max(hi16(wo0), max(0, c2 + BW2)) : c2;
      const uint32_t cf = __vmaxs2(ci, relu_pack(cw_lo + pbs_lo, cw_hi + pbs_hi));
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
      // diagonal carries into the first node: row i-1 at the last node of the previous virtual warp
      uint32_t cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1);
      if (lane == 0) {
        if (w) {                                   // lo <- v0 (carry 0), hi <- v2 (carry c2)
          cM = xo.x;
          cI = xo.y;
          cD = __vmaxs2(xo.z, relu_pack(0, c2 + K2));
        } else {                                   // lo <- floor, hi <- v1 (carry c1)
          cM = __byte_perm(xo.x, 0u, 0x1054u);
          cI = __byte_perm(xo.y, 0u, 0x1054u);
          cD = __byte_perm(__vmaxs2(xo.z, relu_pack(c1 + K1, 0)), 0u, 0x1054u);
        }
      }
      mp[0] = __viaddmax_s16x2(cM, tMM[0], mp[0]);
      mp[0] = __viaddmax_s16x2(cI, tIM[0], mp[0]);
      // ---------------- phase B: M(i, .) (Alg 2 l.16 + emission, reading R15), row max, D chain
      {
        uint32_t e[Q];
        if (x < 20 || x == 26) {
          load_row<NT, Q>(tab + (x < 20 ? x : 20) * ROWW, g, e);     // shared memory
        } else {
          load_row<NT, Q>(reinterpret_cast<const uint32_t*>(a.rsc) + x * ROWW, g, e);   // rare codes: L2
        }
#pragma unroll
        for (int q = Q - 1; q >= 0; --q) {
          const uint32_t m = __viaddmax_s16x2(q ? Dc[q - 1] : cD, tDM[q], mp[q]);
          Mc[q] = __viaddmax_s16x2_relu(m, e[q], e[q]);
        }
      }
#pragma unroll
      for (int q = 0; q + 1 < Q; q += 2) R = __vimax3_s16x2(R, Mc[q], Mc[q + 1]);
      if constexpr (Q % 2) R = __vmaxs2(R, Mc[Q - 1]);
      Dc[0] = 0u;
#pragma unroll
      for (int q = 1; q < Q; ++q)
        Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], __viaddmax_s16x2_relu(Mc[q - 1], tMD[q - 1], tMD[q - 1]));
      const uint32_t cl =
          __viaddmax_s16x2(Dc[Q - 1], tDD[Q - 1], __viaddmax_s16x2_relu(Mc[Q - 1], tMD[Q - 1], tMD[Q - 1]));
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
      const bool hit = __any_sync(0xffffffffu, (__vadd2(R, (uint32_t)(0x8000 - thr) * 0x10001u) & 0x80008000u) != 0u);
      if (lane == 31)
        xcs[par * 2 + w] = make_uint4(Mc[Q - 1], Ic[Q - 1], __vmaxs2(Dc[Q - 1], __viaddmax_s16x2_relu(ci, s31p, s31p)),
                                      out | (hit ? 0x80000000u : 0u));
      bar_arrive(bmine + par, 2 * 32);
      pending = true;
      par ^= 1;
     }
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
