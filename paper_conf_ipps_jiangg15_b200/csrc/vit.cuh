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

// One row of Alg 2 for the G-lane group (lane z owns nodes z*Q+1..z*Q+Q).
// Returns nothing; updates Mc/Ic/Dc in place and the specials.
template <int G, int Q>
struct VitLane {
  int tBM[Q], tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
  int Mc[Q], Ic[Q], Dc[Q];

  __device__ __forceinline__ void row(const int32_t* __restrict__ rrow, int z, int& xB, int& xJ, int& xC,
                                      int move, bool& ovf, bool live) {
    int r[Q];
    load_row<G, Q>(reinterpret_cast<const uint32_t*>(rrow), z, reinterpret_cast<uint32_t(&)[Q]>(r));
    // diagonal carries: row i-1 values at node z*Q, owned by lane z-1 (none for lane 0)
    int cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1, G);
    int cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1, G);
    int cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1, G);
    if (z == 0) cM = cI = cD = kNegW;
    // M and I (Alg 2 l.15-16), descending so that q-1 still holds row i-1
#pragma unroll
    for (int q = Q - 1; q >= 0; --q) {
      const int pm = q ? Mc[q - 1] : cM;
      const int pi = q ? Ic[q - 1] : cI;
      const int pd = q ? Dc[q - 1] : cD;
      int m = sadd(xB, tBM[q]);
      m = __viaddmax_s32(pm, tMM[q], m);
      m = __viaddmax_s32(pi, tIM[q], m);
      m = __viaddmax_s32(pd, tDM[q], m);
      Ic[q] = __viaddmax_s32(Ic[q], tII[q], sadd(Mc[q], tMI[q]));
      Mc[q] = sadd(m, r[q]);                                  // + emission (reading R15)
    }
    int xE = kNegW;
#pragma unroll
    for (int q = 0; q + 1 < Q; q += 2) xE = __vimax3_s32(xE, Mc[q], Mc[q + 1]);
    if constexpr (Q % 2) xE = max(xE, Mc[Q - 1]);
    // D: partial from M (Alg 2 l.17, reading R16) fused with the in-lane D->D chain
    Dc[0] = kNegW;
#pragma unroll
    for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], sadd(Mc[q - 1], tMD[q - 1]));
    // xE over the group (Alg 2 l.22) and the specials (l.24; reading R17)
    if constexpr (G == 32) {
      xE = __reduce_max_sync(0xffffffffu, xE);
    } else {
#pragma unroll
      for (int o = G / 2; o >= 1; o >>= 1) xE = max(xE, __shfl_xor_sync(0xffffffffu, xE, o));
    }
    if (live && !ovf) {
      if (xE >= 32767) {
        ovf = true;
      } else {
        xC = max(xC, xE - 500);
        xJ = max(xJ, xE - 500);
        xB = max(xJ, kBaseW) + move;
      }
    }
    // Lazy-F across lane boundaries (l.25, Fig 7): each lane's outgoing D (+DD) feeds the
    // next lane's first node; walk while it improves; repeat while any lane improved.
    int cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], sadd(Mc[Q - 1], tMD[Q - 1]));
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

  VitLane<G, Q> V;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = z * Q + q;   // node z*Q + q + 1: into-k BM MM IM DM, out-of-k MD MI II DD
    V.tBM[q] = a.tr[0 * G * Q + o];
    V.tMM[q] = a.tr[1 * G * Q + o];
    V.tIM[q] = a.tr[2 * G * Q + o];
    V.tDM[q] = a.tr[3 * G * Q + o];
    V.tMD[q] = a.tr[4 * G * Q + o];
    V.tMI[q] = a.tr[5 * G * Q + o];
    V.tII[q] = a.tr[6 * G * Q + o];
    V.tDD[q] = a.tr[7 * G * Q + o];
  }
  const long long ntot = a.list ? *a.nlist : a.nseq;

  for (;;) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(a.counter, (unsigned long long)NG);
    base = __shfl_sync(0xffffffffu, base, 0);
    if ((long long)base >= ntot) break;
    const long long idx = (long long)base + grp;
    bool valid = idx < ntot;
    const int s = valid ? (a.list ? a.list[idx] : (int)idx) : 0;
    if (valid && a.done && a.done[s]) valid = false;    // already scored by the pipeline long lane
    const int L = valid ? a.len[s] : 0;
    int Lmax = L;
#pragma unroll
    for (int o = 16; o >= G; o >>= 1) Lmax = max(Lmax, __shfl_xor_sync(0xffffffffu, Lmax, o));
    const uint32_t* wp = a.words + (valid ? (size_t)a.woff16[s] * 4 : 0);
    const int nw = (L + 5) / 6;
    const int move = valid ? a.move[L] : 0;

#pragma unroll
    for (int q = 0; q < Q; ++q) V.Mc[q] = V.Ic[q] = V.Dc[q] = kNegW;      // Alg 2 l.9
    int xB = kBaseW + move, xJ = kNegW, xC = kNegW;
    bool ovf = false;

    const int nblk = (Lmax + 5) / 6;
    uint32_t wnext = (0 < nw) ? __ldg(wp) : 0xffffffffu;
    for (int blk = 0; blk < nblk; ++blk) {
      const uint32_t w = wnext;
      wnext = (blk + 1 < nw) ? __ldg(wp + blk + 1) : 0xffffffffu;
#pragma unroll
      for (int j = 0; j < 6; ++j) {
        const int x = (w >> (5 * j)) & 31;          // 31: past the end of this sequence
        V.row(sm + x * ROWW, z, xB, xJ, xC, move, ovf, x != kPadCode);
      }
    }
    if (valid && z == 0) a.raw_sorted[s] = (int16_t)(ovf ? 32767 : xC);
  }
}

}  // namespace hmg
