// vit_pair.cuh -- Viterbi filter (Alg 2, + Lazy-F, P:519-533 / Fig 7) with TWO DP
// cells per 32-bit register: s16x2 DPX, half the instructions of the s32 kernels (vit.cuh).
//
// Layout: HMMER's Farrar striping (ref [19] P:1344-1346) over 2G "virtual lanes", as in the MSV
// kernel: virtual lane v owns the contiguous nodes v*Q+1 .. v*Q+Q; register q of lane z holds
// node z*Q+q+1 in its low half and node (z+G)*Q+q+1 in its high half.  The diagonal carry and the
// D->D carry between virtual lanes are one __shfl_sync + PRMT (lane 0's high half takes lane
// G-1's low half).
//
// Offset arithmetic.  HMMER's word cells saturate at -32768; a 16-bit lane
// cannot hold a value and also absorb an add of a transition as low as -32768 without wrapping.
// So each sequence gets a floor F = sat16(xN + move(L) + min_k tBM_k) <= every B->M term, and
// cells are stored as v' = max(v, F) - F in [0, 32767].  Every HMMER op maps to one DPX op:
//     sat(a + t), t <= 0   ->  VIADDMNMX.S16x2(a', t, 0)     = max(a' + t, 0)
//     max(Bk, ...)         ->  Bk' = Bk - F >= 0 as the third operand
// and the result of every cell is max(HMMER value, F) - F (proof in DESIGN.md: t <= 0 commutes
// with the floor; the M max always contains Bk >= F, so the emission add sees the exact value).
// The row max xE is therefore exact whenever it is above F, i.e. whenever the running max R' > 0
// at the end; otherwise (rows of -inf emissions only) the sequence is re-scored by the s32 kernel.
// The top: a cell plus the largest emission must stay <= 32767, i.e. R' <= safe = 32767 - rmax
// and Bk' <= safe.  The window follows the scores: on a hit row (xB rises with xJ) the floor is
// raised to F' = sat16(xB + min_k tBM_k), still <= every B->M term, and every cell is re-based
// (v' <- max(v' - (F' - F), 0), the same map), so strong hits and overflow (xE >= 32767,
// reading R17) are scored exactly in the window.  Left to the s32 kernel (device redo list):
// sequences whose every row stays at the floor (rows of -inf emissions only) and any that would
// leave the window within one run of rows (not seen on Dirichlet profiles).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"
#include "msv.cuh"   // Chunks / load_row / ResStream

namespace hmg {

constexpr int kRedo = -65536;   // finish(): not a word score (those are >= -32768)

// SCAN: resolve the cross-lane D->D carries with one max-plus
// prefix scan over the lanes (log2 G shuffle steps on (carry, tDD cost) pairs, both halves at
// once, then the low -> high wrap) instead of vote-terminated passes.  A span of lanes maps an
// incoming carry c to max(A, relu(c - C)) with C = -(sum of its tDD); spans compose as
// (A1, C1) then (A2, C2) -> (max(A2, relu(A1 - C2)), C1 + C2).  Costs are kept as u16 clamped at
// 32767 (exact: carries are <= 32767, so any larger cost yields the floor), added with one
// VIADDMNMX.U16x2 min -- no wrap-around.  Same fixed point as the passes.
template <int G, int Q, bool SCAN = false>
struct VitPairLane {
  uint32_t tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];   // s16x2 transitions
  uint32_t bcost;            // SCAN: -(sum of the lane's tDD) per half, u16 clamped at 32767
  uint32_t Mc[Q], Ic[Q], Dc[Q], Bk[Q];                              // s16x2 cells (offset by F)
  uint32_t R;                // running max of M' over the rows
  uint32_t thrv;             // 0x8000 - threshold, per half: vote fires when R' >= threshold
  int F, xJ, move, safe, tbm_min;
  int state;                 // 0 running, 1 overflow (raw 32767), 2 re-score with the s32 kernel

  __device__ __forceinline__ void load(const uint32_t* __restrict__ tr, int z) {
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int o = z * Q + q;    // [8][G][Q] words: BM MM IM DM MD MI II DD
      tMM[q] = tr[1 * G * Q + o];
      tIM[q] = tr[2 * G * Q + o];
      tDM[q] = tr[3 * G * Q + o];
      tMD[q] = tr[4 * G * Q + o];
      tMI[q] = tr[5 * G * Q + o];
      tII[q] = tr[6 * G * Q + o];
      tDD[q] = tr[7 * G * Q + o];
    }
    int clo = 0, chi = 0;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      clo = min(32767, clo - (int)(int16_t)(tDD[q] & 0xffffu));
      chi = min(32767, chi - (int)(int16_t)(tDD[q] >> 16));
    }
    bcost = (uint32_t)clo | ((uint32_t)chi << 16);
  }

  // Bk' = sat16(xB + tBM_k) - F for both halves; false if a term exceeds the safe bound
  __device__ __forceinline__ bool set_bk(const uint32_t* __restrict__ tbm, int z, int xB) {
    bool okv = true;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const uint32_t w = __ldg(tbm + z * Q + q);
      const int lo = max(-32768, min(32767, xB + (int)(int16_t)(w & 0xffffu))) - F;
      const int hi = max(-32768, min(32767, xB + (int)(int16_t)(w >> 16))) - F;
      okv = okv && lo <= safe && hi <= safe;
      Bk[q] = (uint32_t)max(lo, 0) | ((uint32_t)max(hi, 0) << 16);
    }
    return okv;
  }

  __device__ __forceinline__ void set_thr(int thr) {       // thr: HMMER-scale hit threshold
    const int t = min(thr - F, safe + 1);                   // >= 1: F <= xN + move < thr
    thrv = (uint32_t)(0x8000 - t) * 0x10001u;
  }

  __device__ __forceinline__ void kill() {                 // state != 0: cells pinned at the floor
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = Bk[q] = 0u;
    R = 0u;
    thrv = 0x80008000u;                                     // the vote fires every row
  }

  // raise the floor by d >= 0: v' <- max(v' - d, 0) on every live value (the same floor map)
  __device__ __forceinline__ void rebase(int d, uint32_t& cout) {
    if (d <= 0) return;
    const uint32_t n = d >= 32768 ? 0x80008000u : (uint32_t)(uint16_t)(-d) * 0x10001u;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      Mc[q] = __viaddmax_s16x2_relu(Mc[q], n, n);
      Ic[q] = __viaddmax_s16x2_relu(Ic[q], n, n);
      Dc[q] = __viaddmax_s16x2_relu(Dc[q], n, n);
    }
    R = __viaddmax_s16x2_relu(R, n, n);
    cout = __viaddmax_s16x2_relu(cout, n, n);
  }

  __device__ __forceinline__ void start(const uint32_t* __restrict__ tbm, int z, int mv, int tmin, int sf,
                                        bool valid, unsigned gbits) {
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = 0u;   // Alg 2 l.9: -inf -> floor
    R = 0u;
    move = mv;
    tbm_min = tmin;
    F = max(-32768, kBaseW + mv + tmin);                        // <= sat16(xN + move + tBM_k)
    safe = sf;
    xJ = kNegW;
    state = valid ? 0 : 1;
    const bool okv = set_bk(tbm, z, kBaseW + move);            // xB = xN + N->B
    const bool bad = (__ballot_sync(0xffffffffu, !okv) & gbits) != 0u;
    if (valid && bad) state = 2;
    if (state) {
      kill();
      if (!valid) thrv = 0u;                                  // idle group: never votes
    } else {
      set_thr(min(kBaseW + 501, 32767));
    }
  }

  // Alg 2 l.15-20 for one row from the diagonal carries (cM, cI, cD: row i-1 at the last node of the
  // previous virtual lane): M, I, the running max R, and D with its in-lane D->D chain; returns the
  // lane's outgoing D carry (D (+) tDD at its last node)
  __device__ __forceinline__ uint32_t cells(const uint32_t (&e)[Q], uint32_t cM, uint32_t cI, uint32_t cD) {
    // M and I (Alg 2 l.15-16, emission per reading R15), descending: q-1 still holds row i-1
#pragma unroll
    for (int q = Q - 1; q >= 0; --q) {
      const uint32_t pm = q ? Mc[q - 1] : cM;
      const uint32_t pi = q ? Ic[q - 1] : cI;
      const uint32_t pd = q ? Dc[q - 1] : cD;
      uint32_t m = __viaddmax_s16x2(pm, tMM[q], Bk[q]);
      m = __viaddmax_s16x2(pi, tIM[q], m);
      m = __viaddmax_s16x2(pd, tDM[q], m);
      // max(a + t, 0) as VIADDMNMX.RELU(a, t, t): t <= 0 never wins; for the emission,
      // m >= Bk' >= 0 so m + e >= e (no zero register needed)
      Ic[q] = __viaddmax_s16x2(Ic[q], tII[q], __viaddmax_s16x2_relu(Mc[q], tMI[q], tMI[q]));
      Mc[q] = __viaddmax_s16x2_relu(m, e[q], e[q]);
    }
#pragma unroll
    for (int q = 0; q + 1 < Q; q += 2) R = __vimax3_s16x2(R, Mc[q], Mc[q + 1]);
    if constexpr (Q % 2) R = __vmaxs2(R, Mc[Q - 1]);
    // D: partial from M (l.17, reading R16) fused with the in-lane D->D chain
    Dc[0] = 0u;
#pragma unroll
    for (int q = 1; q < Q; ++q)
      Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], __viaddmax_s16x2_relu(Mc[q - 1], tMD[q - 1], tMD[q - 1]));
    return __viaddmax_s16x2(Dc[Q - 1], tDD[Q - 1], __viaddmax_s16x2_relu(Mc[Q - 1], tMD[Q - 1], tMD[Q - 1]));
  }

  __device__ __forceinline__ bool hit_vote() const { return (__vadd2(R, thrv) & 0x80008000u) != 0u; }

  // a row whose running max reached the threshold (ballot bal != 0): Alg 2 l.22-24 -- E->J, J->B,
  // the floor raised and every cell re-based, or overflow / the s32 re-score
  __device__ __forceinline__ void on_hit(unsigned bal, const uint32_t* __restrict__ tbm, int z, unsigned gbits,
                                         uint32_t& cout) {
    uint32_t mm = R;
#pragma unroll
    for (int o = G / 2; o >= 1; o >>= 1) mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, o));
    const int mp = max((int)(mm & 0xffffu), (int)(mm >> 16));
    bool mine = (bal & gbits) != 0u && state == 0;
    bool okv = true;
    if (mine) {
      if (mp > safe) {
        state = 2;                                  // beyond the 16-bit window: s32 re-score
      } else if (mp + F >= 32767) {
        state = 1;                                  // reading R17: overflow -> +inf, pass
      } else {
        xJ = mp + F - 500;                          // E->J (and E->C: xC == xJ)
        const int xB = max(xJ, kBaseW) + move;
        const int Fn = max(-32768, min(32767, xB + tbm_min));
        rebase(Fn - F, cout);
        F = Fn;
        okv = set_bk(tbm, z, xB);
        set_thr(min(max(xJ, kBaseW) + 501, 32767));
      }
    }
    const bool bad = (__ballot_sync(0xffffffffu, !okv) & gbits) != 0u;
    if (mine && bad) state = 2;
    if ((bal & gbits) && state) kill();
  }

  // Lazy-F across virtual lanes (l.25, Fig 7): passes while any carry improves (reading R19)
  __device__ __forceinline__ void lazy(uint32_t cout, int src, uint32_t sel) {
    for (;;) {
      uint32_t cin = __shfl_sync(0xffffffffu, cout, src, G);
      cin = __byte_perm(cin, 0u, sel);
      bool imp = __vmaxs2(cin, Dc[0]) != Dc[0];
      if (!__any_sync(0xffffffffu, imp)) break;
      Dc[0] = __vmaxs2(Dc[0], cin);
      constexpr int K0 = Q < 3 ? Q : 3;      // most D->D runs die within a few nodes
#pragma unroll
      for (int q = 1; q < K0; ++q) {
        const uint32_t nd = __viaddmax_s16x2_relu(Dc[q - 1], tDD[q - 1], tDD[q - 1]);
        imp = imp && (__vmaxs2(nd, Dc[q]) != Dc[q]);
        Dc[q] = __vmaxs2(Dc[q], nd);
      }
      if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
        for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], Dc[q]);
        cout = __viaddmax_s16x2(Dc[Q - 1], tDD[Q - 1], cout);
      } else {
        break;
      }
    }
  }

  __device__ __forceinline__ void row(const uint32_t* __restrict__ rrow, const uint32_t* __restrict__ tbm, int z,
                                      unsigned gbits) {
    const uint32_t sel = (z == 0) ? 0x1054u : 0x3210u;   // lane 0: low <- floor, high <- lane G-1 low
    const int src = (z + G - 1) & (G - 1);
    uint32_t e[Q];
    load_row<G, Q>(rrow, z, e);
    // diagonal carries: row i-1 at the last node of the previous virtual lane
    uint32_t cM = __shfl_sync(0xffffffffu, Mc[Q - 1], src, G);
    uint32_t cI = __shfl_sync(0xffffffffu, Ic[Q - 1], src, G);
    uint32_t cD = __shfl_sync(0xffffffffu, Dc[Q - 1], src, G);
    cM = __byte_perm(cM, 0u, sel);
    cI = __byte_perm(cI, 0u, sel);
    cD = __byte_perm(cD, 0u, sel);
    uint32_t cout = cells(e, cM, cI, cD);
    // hit / overflow / safe-bound vote (Alg 2 l.22-24 on the rows that need it)
    const unsigned bal = __ballot_sync(0xffffffffu, hit_vote());
    if (bal) on_hit(bal, tbm, z, gbits, cout);
    if constexpr (SCAN) {
      // inclusive max-plus scan of (carry out, tDD cost) over the lanes, both halves
      uint32_t c = cout, sm = bcost;
#pragma unroll
      for (int d = 1; d < G; d <<= 1) {
        const uint32_t c2 = __shfl_up_sync(0xffffffffu, c, d, G);
        const uint32_t s2 = __shfl_up_sync(0xffffffffu, sm, d, G);
        if (z >= d) {
          c = __vimax_s16x2_relu(c, __vsub2(c2, sm));          // max(c, relu(c2 - cost))
          sm = __viaddmin_u16x2(s2, sm, 0x7fff7fffu);           // cost sum, clamped
        }
      }
      uint32_t cex = __shfl_up_sync(0xffffffffu, c, 1, G);
      uint32_t sex = __shfl_up_sync(0xffffffffu, sm, 1, G);
      const uint32_t wrap = __shfl_sync(0xffffffffu, c, G - 1, G) << 16;   // low chain out -> high
      if (z == 0) cex = sex = 0u;
      const uint32_t cin = __vimax_s16x2_relu(cex, __vsub2(wrap, sex));     // high: max(c, relu(wrap - C))
      bool imp = __vmaxs2(cin, Dc[0]) != Dc[0];
      if (__any_sync(0xffffffffu, imp)) {
        Dc[0] = __vmaxs2(Dc[0], cin);
        constexpr int K0 = Q < 3 ? Q : 3;
#pragma unroll
        for (int q = 1; q < K0; ++q) {
          const uint32_t nd = __viaddmax_s16x2_relu(Dc[q - 1], tDD[q - 1], tDD[q - 1]);
          imp = imp && (__vmaxs2(nd, Dc[q]) != Dc[q]);
          Dc[q] = __vmaxs2(Dc[q], nd);
        }
        if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
          for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], Dc[q]);
        }
      }
      return;
    }
    lazy(cout, src, sel);
  }

  // raw xC (== xJ) = max over rows of xE - 500; 32767 on overflow; kRedo (re-score) when the
  // result is not exact in the 16-bit window
  __device__ __forceinline__ int finish() {
    uint32_t mm = R;
#pragma unroll
    for (int o = G / 2; o >= 1; o >>= 1) mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, o));
    const int mp = max((int)(mm & 0xffffu), (int)(mm >> 16));
    if (state == 1) return 32767;
    if (state == 2) return kRedo;
    if (mp > 0) return max(xJ, max(kNegW, mp + F - 500));   // rows before the last re-base: xJ
    return xJ > kNegW ? xJ : kRedo;    // later rows all <= F <= xJ; never above the floor: redo

  }
};

// (a register cap for more resident warps -- 96 / 80 / 64 registers -- measured 13% / 77% / 200%
//  slower on the config-3 Viterbi stage: the row state spills; profiles/vit_minb_r01.jsonl)
template <int G, int Q, bool SCAN = false>
__global__ void __launch_bounds__(128) vit_pair_kernel(const VitArgs a) {
  constexpr int ROWW = Q * G;              // s16x2 words per residue row
  constexpr int NG = 32 / G;
  extern __shared__ uint4 smem4[];
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    const int n4 = (kRows * ROWW + 3) / 4;
    for (int i = threadIdx.x; i < n4; i += blockDim.x) smem4[i] = src[i];
  }
  __syncthreads();
  const uint32_t* sm = reinterpret_cast<const uint32_t*>(smem4);
  const uint32_t* tr = reinterpret_cast<const uint32_t*>(a.tr);

  const int lane = threadIdx.x & 31;
  const int z = lane & (G - 1);
  const int grp = lane / G;

  VitPairLane<G, Q, SCAN> V;
  V.load(tr, z);
  const unsigned gbits = (G == 32 ? 0xffffffffu : ((1u << G) - 1u)) << (grp * G);
  const long long ntot = a.list ? *a.nlist : a.nseq;

  for (;;) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(a.counter, (unsigned long long)NG);
    base = __shfl_sync(0xffffffffu, base, 0);
    if ((long long)base >= ntot) break;
    const long long idx = (long long)base + grp;
    bool valid = idx < ntot;
    const int s = valid ? (a.list ? a.list[idx] : (int)idx) : 0;
    if (valid && s < a.ndone && a.done[s]) valid = false;    // already scored by the pipeline long lane
    const int L = valid ? a.len[s] : 0;
    int Lmax = L;
#pragma unroll
    for (int o = 16; o >= G; o >>= 1) Lmax = max(Lmax, __shfl_xor_sync(0xffffffffu, Lmax, o));
    const uint32_t* wp = a.words + (valid ? (size_t)a.woff16[s] * 4 : 0);
    const int nw = (L + 5) / 6;
    const int mv = valid ? a.move[L] : 0;
    V.start(tr, z, mv, a.tbm_min, a.safe, valid, gbits);

    const int nqmax = (Lmax + 23) / 24;
    const int nwmax = (Lmax + 5) / 6;                 // rows stop at the warp's last word
    ResStream rs;
    rs.init(wp, nw);
    for (int iq = 0; iq < nqmax; ++iq) {
      uint4 w4 = rs.next(iq);
#pragma unroll 1
      for (int k = 0; k < 4; ++k) {
        if (iq * 4 + k >= nwmax) break;               // warp-uniform (Lmax is the warp's max)
        const uint32_t w = w4.x;
        w4.x = w4.y;
        w4.y = w4.z;
        w4.z = w4.w;
#pragma unroll        // (one row per iteration: config 3 -4%, M = 500 +10%, M = 100 +7%; cmp_r02zzh.jsonl)
        for (int j = 0; j < 6; ++j) {
          const int x = (w >> (5 * j)) & 31;          // 31 (pad): -inf emissions, cells decay
          V.row(sm + x * ROWW, tr, z, gbits);
        }
      }
    }
    const int raw = V.finish();
    if (valid && z == 0) {
      if (raw >= -32768) {
        a.raw_sorted[s] = (int16_t)raw;
      } else {
        const unsigned long long k = atomicAdd(a.redo_count, 1ull);
        a.redo_list[k] = s;
      }
    }
  }
}

}  // namespace hmg
