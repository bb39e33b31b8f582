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

template <int G, int Q>
__global__ void __launch_bounds__(128) vit_reg_kernel(const VitArgs a) {
  constexpr int Q2 = (Q + 1) / 2;          // s16 emission pairs per lane
  constexpr int ROWW = Q2 * G;             // words per residue row
  constexpr int NG = 32 / G;
  extern __shared__ uint4 smem4[];
  uint32_t* sm = reinterpret_cast<uint32_t*>(smem4);
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    const int n4 = (kRows * ROWW + 3) / 4;
    for (int i = threadIdx.x; i < n4; i += blockDim.x) smem4[i] = src[i];
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const int z = lane & (G - 1);
  const int grp = lane / G;
  const unsigned gbits = (G == 32 ? 0xffffffffu : ((1u << G) - 1u)) << (grp * G);

  // this lane's transitions, s32, node k = z*Q + q + 1 (into-k: BM MM IM DM; out-of-k: MD MI II DD)
  int tBM[Q], tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = z * Q + q;
    tBM[q] = a.tr[0 * G * Q + o];
    tMM[q] = a.tr[1 * G * Q + o];
    tIM[q] = a.tr[2 * G * Q + o];
    tDM[q] = a.tr[3 * G * Q + o];
    tMD[q] = a.tr[4 * G * Q + o];
    tMI[q] = a.tr[5 * G * Q + o];
    tII[q] = a.tr[6 * G * Q + o];
    tDD[q] = a.tr[7 * G * Q + o];
  }
  const long long ntot = a.list ? *a.nlist : a.nseq;

  for (;;) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(a.counter, (unsigned long long)NG);
    base = __shfl_sync(0xffffffffu, base, 0);
    if ((long long)base >= ntot) break;
    const long long idx = (long long)base + grp;
    const bool valid = idx < ntot;
    const int s = valid ? (a.list ? a.list[idx] : (int)idx) : 0;
    const int L = valid ? a.len[s] : 0;
    int Lmax = L;
#pragma unroll
    for (int o = 16; o >= G; o >>= 1) Lmax = max(Lmax, __shfl_xor_sync(0xffffffffu, Lmax, o));
    const uint32_t* wp = a.words + (valid ? (size_t)a.woff16[s] * 4 : 0);
    const int nw = (L + 5) / 6;
    const int move = valid ? a.move[L] : 0;

    int Mc[Q], Ic[Q], Dc[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = kNegW;      // Alg 2 l.9
    const int xN = kBaseW;
    int xB = xN + move, xJ = kNegW, xC = kNegW;
    bool ovf = false, done = !valid;

    const int nblk = (Lmax + 5) / 6;
    uint32_t wnext = (0 < nw) ? __ldg(wp) : 0xffffffffu;
    for (int blk = 0; blk < nblk; ++blk) {
      const uint32_t w = wnext;
      wnext = (blk + 1 < nw) ? __ldg(wp + blk + 1) : 0xffffffffu;
#pragma unroll 1
      for (int j = 0; j < 6; ++j) {
        const int x = (w >> (5 * j)) & 31;
        if (x == kPadCode) done = true;                 // past the end of this sequence
        uint32_t e2[Q2];
        load_row<G, Q2>(sm + x * ROWW, z, e2);
        // diagonal carries (row i-1 values at node z*Q, owned by lane z-1)
        int cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1, G);
        int cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1, G);
        int cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1, G);
        if (z == 0) cM = cI = cD = kNegW;
        int xE = kNegW;
        // M and I, descending so that q-1 still holds row i-1 (Alg 2 l.15-16)
#pragma unroll
        for (int q = Q - 1; q >= 0; --q) {
          const int pm = q ? Mc[q - 1] : cM;
          const int pi = q ? Ic[q - 1] : cI;
          const int pd = q ? Dc[q - 1] : cD;
          const int r = (q & 1) ? ((int)e2[q >> 1] >> 16) : (int)(int16_t)(e2[q >> 1] & 0xffffu);
          int m = sadd(xB, tBM[q]);
          m = __viaddmax_s32(pm, tMM[q], m);
          m = __viaddmax_s32(pi, tIM[q], m);
          m = __viaddmax_s32(pd, tDM[q], m);
          m = sadd(m, r);                                       // + emission (reading R15)
          const int in = __viaddmax_s32(Ic[q], tII[q], sadd(Mc[q], tMI[q]));
          Mc[q] = m;
          Ic[q] = in;
        }
#pragma unroll
        for (int q = 0; q + 1 < Q; q += 2) xE = __vimax3_s32(xE, Mc[q], Mc[q + 1]);
        if constexpr (Q % 2) xE = max(xE, Mc[Q - 1]);
        // D: partial from M (Alg 2 l.17, reading R16) fused with the in-lane D->D chain
        Dc[0] = kNegW;
#pragma unroll
        for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], sadd(Mc[q - 1], tMD[q - 1]));
        // group max of xE (Alg 2 l.22)
        if constexpr (G == 32) {
          xE = __reduce_max_sync(0xffffffffu, xE);
        } else {
#pragma unroll
          for (int o = G / 2; o >= 1; o >>= 1) xE = max(xE, __shfl_xor_sync(0xffffffffu, xE, o));
        }
        // specials (Alg 2 l.24; reading R17)
        if (!done && !ovf) {
          if (xE >= 32767) {
            ovf = true;
          } else {
            xC = max(xC, xE - 500);
            xJ = max(xJ, xE - 500);
            xB = max(xJ, xN) + move;
          }
        }
        // Lazy-F across lane boundaries (Alg 2 l.25; Fig 7)
        int cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], sadd(Mc[Q - 1], tMD[Q - 1]));
        for (;;) {
          int cin = __shfl_up_sync(0xffffffffu, cout, 1, G);
          if (z == 0) cin = kNegW;
          const bool imp = cin > Dc[0];
          if (!__any_sync(0xffffffffu, imp)) break;
          if (imp) {
            Dc[0] = cin;
#pragma unroll
            for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], Dc[q]);
            cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], cout);
          }
        }
      }
    }
    if (valid && z == 0) a.raw_sorted[s] = (int16_t)(ovf ? 32767 : xC);
  }
}

}  // namespace hmg
