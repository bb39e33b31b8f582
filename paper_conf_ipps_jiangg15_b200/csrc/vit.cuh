// vit.cuh -- Viterbi-filter kernel for sm_100a (Alg 2) with
// warp-synchronous Lazy-F.
//
// vit_reg_kernel<G, Q>: a group of G lanes scores one sequence, 32/G sequences
// per warp (the paper's warp-per-sequence, generalised).  Lane z
// owns the CONTIGUOUS node block k = z*Q+1 .. z*Q+Q (Farrar's stripe mapped
// onto lanes, ref [19] P:1344-1346) with M, I, D cells and the lane's 8
// transition vectors in registers as s32.  Every 16-bit saturating add of
// HMMER's word system (sat(a+b) = max(a+b, -32768)) is ONE DPX instruction
// (VIADDMNMX); the upper clamp is never needed because any M cell >= 32767
// is an overflow of the row (reading R17) and all transitions are <= 0.
//
// D->D (Lazy-F): the in-lane part of the D chain is fused into the row pass
// (D_{k+1} = max(M_k + tMD_k, D_k + tDD_k), one more VIADDMNMX per cell).
// What remains is the carry across lane boundaries: each lane passes its
// outgoing D (+tDD) to the next lane with __shfl_up_sync, applies it to its
// block, and the passes repeat until __any_sync says no lane's carry improved
// -- the paper's "__all(MD > DD)" termination (Fig 7) read as
// "stop when no DD candidate strictly improves" (reading R19).  By
// max-plus monotonicity this reaches the same fixed point as the sequential
// closure the oracle performs (Lazy-F exactness).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"
#include "msv.cuh"   // Chunks / load_row

namespace hmg {

__device__ __forceinline__ int sadd(int a, int b) { return __viaddmax_s32(a, b, kNegW); }  // max(a+b, -32768)

// State of one lane of a G-lane group (lane z owns nodes z*Q+1..z*Q+Q) and one row of Alg 2.
//
// xB speculation: xB = max(xJ, xN) + move changes only on rows whose best
// M cell exceeds max(xJ, xN) + 500 (a hit) or overflows.  The B->M_k terms
// Bk[q] = sat(xB + tBM) are therefore kept in registers, xE is tracked as a running max R
// (xC == xJ == max over rows of xE - 500), and one __ballot_sync per row detects the rows
// where xB must change; only then is R reduced over the group and Bk recomputed.
// LAT (long lane): the lane's outgoing D carry is computed directly from the M cells
// (max_q M_q + w_q, w_q = tMD_q + sum of the later tDD) instead of waiting for the in-lane
// D chain, shortening the row's critical path; cross-lane passes then move only carries.
template <int G, int Q, bool LAT>
struct VitLane {
  int tBM[Q], tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
  int wout[LAT ? Q : 1];   // LAT: tMD_q + sum_{m>q} tDD_m
  int bsum;                // sum of the lane's tDD (carry through the whole block)
  int Mc[Q], Ic[Q], Dc[Q], Bk[Q];
  int R0, R1;              // running max of M over the rows (two accumulators)
  int xJ, thr, move;
  bool ovf;

  __device__ __forceinline__ void load(const int32_t* __restrict__ tr, int z) {
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int o = z * Q + q;   // node z*Q + q + 1: into-k BM MM IM DM, out-of-k MD MI II DD
      tBM[q] = tr[0 * G * Q + o];
      tMM[q] = tr[1 * G * Q + o];
      tIM[q] = tr[2 * G * Q + o];
      tDM[q] = tr[3 * G * Q + o];
      tMD[q] = tr[4 * G * Q + o];
      tMI[q] = tr[5 * G * Q + o];
      tII[q] = tr[6 * G * Q + o];
      tDD[q] = tr[7 * G * Q + o];
    }
    int acc = 0;
#pragma unroll
    for (int q = Q - 1; q >= 0; --q) {
      if constexpr (LAT) wout[q] = tMD[q] + acc;
      acc += tDD[q];
    }
    bsum = acc;
  }

  __device__ __forceinline__ void start(int mv, bool valid) {
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = kNegW;     // Alg 2 l.9
    move = mv;
    xJ = kNegW;
    ovf = !valid;
    R0 = R1 = kNegW;
    const int xB = kBaseW + move;                                   // xN + N->B
#pragma unroll
    for (int q = 0; q < Q; ++q) Bk[q] = sadd(xB, tBM[q]);
    thr = valid ? min(kBaseW + 501, 32767) : 0x7fffffff;            // xE > max(xJ, xN) + 500
  }

  __device__ __forceinline__ void row(const int32_t* __restrict__ rrow, int z, unsigned gbits) {
    int r[Q];
    load_row<G, Q>(reinterpret_cast<const uint32_t*>(rrow), z, reinterpret_cast<uint32_t(&)[Q]>(r));
    // diagonal carries: row i-1 values at node z*Q, owned by lane z-1 (none for lane 0)
    int cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1, G);
    int cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1, G);
    int cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1, G);
    if (z == 0) cM = cI = cD = kNegW;
    // M and I (Alg 2 l.15-16, + emission per reading R15), descending: q-1 still holds row i-1
#pragma unroll
    for (int q = Q - 1; q >= 0; --q) {
      const int pm = q ? Mc[q - 1] : cM;
      const int pi = q ? Ic[q - 1] : cI;
      const int pd = q ? Dc[q - 1] : cD;
      int m = __viaddmax_s32(pm, tMM[q], Bk[q]);
      m = __viaddmax_s32(pi, tIM[q], m);
      m = __viaddmax_s32(pd, tDM[q], m);
      Ic[q] = __viaddmax_s32(Ic[q], tII[q], sadd(Mc[q], tMI[q]));
      Mc[q] = sadd(m, r[q]);
    }
#pragma unroll
    for (int q = 0; q < Q; q += 4) {
      R0 = __vimax3_s32(R0, Mc[q], (q + 1 < Q) ? Mc[q + 1] : kNegW);
      if (q + 2 < Q) R1 = __vimax3_s32(R1, Mc[q + 2], (q + 3 < Q) ? Mc[q + 3] : kNegW);
    }
    // outgoing D carry of the lane
    int cout;
    if constexpr (LAT) {
      cout = kNegW;
#pragma unroll
      for (int q = 0; q < Q; ++q) cout = __viaddmax_s32(Mc[q], wout[q], cout);
    }
    // D: partial from M (Alg 2 l.17, reading R16) fused with the in-lane D->D chain
    Dc[0] = kNegW;
#pragma unroll
    for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], sadd(Mc[q - 1], tMD[q - 1]));
    if constexpr (!LAT) cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], sadd(Mc[Q - 1], tMD[Q - 1]));
    // hit / overflow vote (Alg 2 l.22-24 only on the rows that need it)
    const bool hit = max(R0, R1) >= thr;
    const unsigned bal = __ballot_sync(0xffffffffu, hit);
    if (bal) {
      int m = max(R0, R1);
      if constexpr (G == 32) {
        m = __reduce_max_sync(0xffffffffu, m);
      } else {
#pragma unroll
        for (int o = G / 2; o >= 1; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
      }
      if ((bal & gbits) && !ovf) {
        if (m >= 32767) {                 // reading R17: overflow -> +inf, pass
          ovf = true;
          thr = 0x7fffffff;
        } else {
          xJ = m - 500;                     // E->J (and E->C: xC == xJ)
          const int xB = max(xJ, kBaseW) + move;
#pragma unroll
          for (int q = 0; q < Q; ++q) Bk[q] = sadd(xB, tBM[q]);
          thr = min(max(xJ, kBaseW) + 501, 32767);
        }
      }
    }
    // Lazy-F across lane boundaries (l.25, Fig 7): the lane's outgoing D feeds the next lane's
    // first node; passes repeat while any lane's incoming carry improves (reading R19).
    if constexpr (LAT) {
      int cin;
      for (;;) {
        cin = __shfl_up_sync(0xffffffffu, cout, 1, G);
        if (z == 0) cin = kNegW;
        const int c2 = max(cout, __viaddmax_s32(cin, bsum, kNegW));
        const bool chg = c2 > cout;
        cout = c2;
        if (!__any_sync(0xffffffffu, chg)) break;
      }
      bool imp = cin > Dc[0];
      if (__any_sync(0xffffffffu, imp)) {
        Dc[0] = max(Dc[0], cin);
        constexpr int K0 = Q < 3 ? Q : 3;
#pragma unroll
        for (int q = 1; q < K0; ++q) {
          const int nd = __viaddmax_s32(Dc[q - 1], tDD[q - 1], kNegW);
          imp = imp && nd > Dc[q];
          Dc[q] = max(Dc[q], nd);
        }
        if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
          for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], Dc[q]);
        }
      }
    } else {
      for (;;) {
        int cin = __shfl_up_sync(0xffffffffu, cout, 1, G);
        if (z == 0) cin = kNegW;
        bool imp = cin > Dc[0];
        if (!__any_sync(0xffffffffu, imp)) break;
        Dc[0] = max(Dc[0], cin);
        constexpr int K0 = Q < 3 ? Q : 3;      // most D->D runs die within a few nodes
#pragma unroll
        for (int q = 1; q < K0; ++q) {
          const int nd = __viaddmax_s32(Dc[q - 1], tDD[q - 1], kNegW);
          imp = imp && nd > Dc[q];
          Dc[q] = max(Dc[q], nd);
        }
        if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
          for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], Dc[q]);
          cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], cout);
        } else {
          break;
        }
      }
    }
  }

  // raw xC (== xJ) of the sequence: max over rows of xE - 500; 32767 on overflow
  __device__ __forceinline__ int finish() {
    int m = max(R0, R1);
    if constexpr (G == 32) {
      m = __reduce_max_sync(0xffffffffu, m);
    } else {
#pragma unroll
      for (int o = G / 2; o >= 1; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
    }
    return ovf ? 32767 : max(kNegW, m - 500);
  }
};

template <int G, int Q>
__global__ void __launch_bounds__(128) vit_reg_kernel(const VitArgs a) {
  constexpr int ROWW = Q * G;              // s32 words per residue row
  constexpr int NG = 32 / G;
  extern __shared__ uint4 smem4[];
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    const int n4 = (kRows * ROWW + 3) / 4;
    for (int i = threadIdx.x; i < n4; i += blockDim.x) smem4[i] = src[i];
  }
  __syncthreads();
  const int32_t* sm = reinterpret_cast<const int32_t*>(smem4);

  const int lane = threadIdx.x & 31;
  const int z = lane & (G - 1);
  const int grp = lane / G;

  VitLane<G, Q, false> V;
  V.load(a.tr, z);
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
    V.start(valid ? a.move[L] : 0, valid);

    const int nqmax = (Lmax + 23) / 24;
    ResStream rs;
    rs.init(wp, nw);
    for (int iq = 0; iq < nqmax; ++iq) {
      uint4 w4 = rs.next(iq);
#pragma unroll 1
      for (int k = 0; k < 4; ++k) {
        const uint32_t w = w4.x;
        w4.x = w4.y;
        w4.y = w4.z;
        w4.z = w4.w;
#pragma unroll
        for (int j = 0; j < 6; ++j) {
          const int x = (w >> (5 * j)) & 31;          // 31 (pad): rows past the end change nothing
          V.row(sm + x * ROWW, z, gbits);
        }
      }
    }
    const int raw = V.finish();
    if (valid && z == 0) a.raw_sorted[s] = (int16_t)raw;
  }
}

}  // namespace hmg
