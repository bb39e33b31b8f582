// vit_cta.cuh -- Viterbi filter (Alg 2 + Lazy-F) with one thread block per sequence.
//
// For long models (M up to 32*W*Q, e.g. 2048 with W = 16 warps x Q = 4 nodes) and for the
// latency-bound longest sequences, W warps cooperate on one DP row: thread g = 32*w + lane
// owns the contiguous nodes g*Q+1 .. g*Q+Q with its 8 transition vectors and M/I/D cells in
// registers (as in vit_reg_kernel).  Per row, besides the intra-warp shuffles:
//   * diagonal carries across warp boundaries: lane 31 of warp w-1 publishes its (M, I, D)
//     for the next row in shared memory (double-buffered by row parity);
//   * Lazy-F across warps (Fig 7): every warp first closes D inside itself, then
//     publishes its outgoing carry; each warp applies its neighbour's carry; rounds repeat
//     while __syncthreads_or says some warp's outgoing carry improved (reading R19);
//   * hits: the running-max xE vote of vit.cuh becomes __syncthreads_or; on a hit row the
//     block reduces xE through shared memory and recomputes the B->M terms.
// Emission scores are s16 pairs in shared memory (32 rows x M x 2 B: 128 KB at M = 2048).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "vit.cuh"

namespace hmg {

template <int W, int Q>
struct VitCtaSmem {
  static constexpr int NT = 32 * W;          // threads = lanes of the DP row
  static constexpr int Q2 = Q / 2;           // s16 emission pairs per lane
  static constexpr int ROWW = Q2 * NT;       // u32 words per residue row
  static constexpr size_t table_bytes = (size_t)kRows * ROWW * 4;
  // shared scratch after the table (ints)
  static constexpr int XC = 0;               // [2][W][3] diagonal carries (M, I, D of lane 31)
  static constexpr int WC = XC + 2 * W * 3;  // [2][W] outgoing D carry of each warp
  static constexpr int RX = WC + 2 * W;      // [W] per-warp xE max on hit rows
  static constexpr int NSCR = RX + W;
};

template <int W, int Q>
__global__ void __launch_bounds__(32 * W) vit_cta_kernel(const VitArgs a) {
  using S = VitCtaSmem<W, Q>;
  static_assert(Q % 2 == 0, "Q must be even (s16 emission pairs)");
  extern __shared__ uint4 smem4[];
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    for (int i = threadIdx.x; i < (int)(S::table_bytes / 16); i += blockDim.x) smem4[i] = src[i];
  }
  uint32_t* tab = reinterpret_cast<uint32_t*>(smem4);
  int* scr = reinterpret_cast<int*>(reinterpret_cast<char*>(smem4) + S::table_bytes);
  __shared__ long long s_next;
  const int g = threadIdx.x;                 // DP lane
  const int w = g >> 5, lane = g & 31;

  // transitions of this thread's nodes (into-k BM MM IM DM, out-of-k MD MI II DD), s32
  int tBM[Q], tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = g * Q + q;
    const int NQ = S::NT * Q;
    tBM[q] = a.tr[0 * NQ + o]; tMM[q] = a.tr[1 * NQ + o]; tIM[q] = a.tr[2 * NQ + o]; tDM[q] = a.tr[3 * NQ + o];
    tMD[q] = a.tr[4 * NQ + o]; tMI[q] = a.tr[5 * NQ + o]; tII[q] = a.tr[6 * NQ + o]; tDD[q] = a.tr[7 * NQ + o];
  }
  __syncthreads();
  const long long ntot = a.list ? *a.nlist : a.nseq;

  for (;;) {
    if (g == 0) s_next = (long long)atomicAdd(a.counter, 1ull);
    __syncthreads();
    const long long idx = s_next;
    __syncthreads();
    if (idx >= ntot) break;
    const int s = a.list ? a.list[idx] : (int)idx;
    if (s < a.ndone && a.done[s]) continue;
    const int L = a.len[s];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    const int move = a.move[L];
    int Mc[Q], Ic[Q], Dc[Q], Bk[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      Mc[q] = Ic[q] = Dc[q] = kNegW;                                  // Alg 2 l.9
      Bk[q] = sadd(kBaseW + move, tBM[q]);
    }
    int R = kNegW, xJ = kNegW;
    bool ovf = false;
    int thr = min(kBaseW + 501, 32767);
    if (lane == 31) {
      scr[S::XC + (0 * W + w) * 3 + 0] = kNegW;
      scr[S::XC + (0 * W + w) * 3 + 1] = kNegW;
      scr[S::XC + (0 * W + w) * 3 + 2] = kNegW;
    }
    __syncthreads();
    int par = 0;                               // row parity (buffer holding row i-1's carries)
    for (int i = 0; i < L; ++i) {
      const int x = (__ldg(wp + i / 6) >> (5 * (i % 6))) & 31;
      // emissions (s16 pairs -> s32)
      uint32_t e2[S::Q2];
      load_row<S::NT, S::Q2>(tab + x * S::ROWW, g, e2);
      int r[Q];
#pragma unroll
      for (int h = 0; h < S::Q2; ++h) {
        r[2 * h] = (int)(int16_t)(e2[h] & 0xffffu);
        r[2 * h + 1] = (int)e2[h] >> 16;
      }
      // diagonal carries (row i-1 at node g*Q): lane l-1, or lane 31 of warp w-1
      int cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1);
      int cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1);
      int cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1);
      if (lane == 0) {
        if (w == 0) {
          cM = cI = cD = kNegW;
        } else {
          const int* xc = scr + S::XC + (par * W + (w - 1)) * 3;
          cM = xc[0];
          cI = xc[1];
          cD = xc[2];
        }
      }
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
      for (int q = 0; q + 1 < Q; q += 2) R = __vimax3_s32(R, Mc[q], Mc[q + 1]);
      // D partial (l.17) + in-thread D->D chain
      Dc[0] = kNegW;
#pragma unroll
      for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], sadd(Mc[q - 1], tMD[q - 1]));
      int cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], sadd(Mc[Q - 1], tMD[Q - 1]));
      // intra-warp Lazy-F with the warp's incoming carry taken as -inf (applied below)
      for (;;) {
        int cin = __shfl_up_sync(0xffffffffu, cout, 1);
        if (lane == 0) cin = kNegW;
        bool imp = cin > Dc[0];
        if (!__any_sync(0xffffffffu, imp)) break;
        if (imp) {
          Dc[0] = cin;
#pragma unroll
          for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], Dc[q]);
          cout = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], cout);
        }
      }
      int rnd = 0;
      if (lane == 31) scr[S::WC + (rnd & 1) * W + w] = cout;
      // hit / overflow (running max, reading R17) joins the first block barrier
      const bool hit = __syncthreads_or(R >= thr);
      if (hit) {
        int m = __reduce_max_sync(0xffffffffu, R);
        if (lane == 0) scr[S::RX + w] = m;
        __syncthreads();
        m = kNegW;
#pragma unroll
        for (int v = 0; v < W; ++v) m = max(m, scr[S::RX + v]);
        if (!ovf) {
          if (m >= 32767) {
            ovf = true;
            thr = 0x7fffffff;
          } else {
            xJ = m - 500;
            const int xB = max(xJ, kBaseW) + move;
#pragma unroll
            for (int q = 0; q < Q; ++q) Bk[q] = sadd(xB, tBM[q]);
            thr = min(max(xJ, kBaseW) + 501, 32767);
          }
        }
      }
      // Lazy-F across warps: apply the left neighbour's outgoing carry, repeat while it changes
      for (;;) {
        int cin = (w > 0) ? scr[S::WC + (rnd & 1) * W + (w - 1)] : kNegW;
        cin = __shfl_sync(0xffffffffu, cin, 0);
        bool changed = false;
        const bool imp = (lane == 0) && cin > Dc[0];
        if (__any_sync(0xffffffffu, imp)) {
          if (imp) Dc[0] = cin;
          for (;;) {                                  // propagate inside the warp
#pragma unroll
            for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], Dc[q]);
            const int c2 = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], cout);
            int cn = __shfl_up_sync(0xffffffffu, c2, 1);
            const bool more = lane > 0 && cn > Dc[0];
            if (more) Dc[0] = cn;
            const bool lane_changed = c2 > cout;
            cout = c2;
            if (lane == 31 && lane_changed) changed = true;
            if (!__any_sync(0xffffffffu, more)) break;
          }
        }
        ++rnd;
        if (lane == 31) {
          scr[S::WC + (rnd & 1) * W + w] = cout;
          const int np = par ^ 1;
          scr[S::XC + (np * W + w) * 3 + 0] = Mc[Q - 1];
          scr[S::XC + (np * W + w) * 3 + 1] = Ic[Q - 1];
          scr[S::XC + (np * W + w) * 3 + 2] = Dc[Q - 1];
        }
        if (!__syncthreads_or(changed)) break;
      }
      par ^= 1;
    }
    // final xC = max over rows of xE - 500 (block max of R)
    {
      int m = __reduce_max_sync(0xffffffffu, R);
      if (lane == 0) scr[S::RX + w] = m;
      __syncthreads();
      m = kNegW;
#pragma unroll
      for (int v = 0; v < W; ++v) m = max(m, scr[S::RX + v]);
      if (g == 0) a.raw_sorted[s] = (int16_t)(ovf ? 32767 : max(kNegW, m - 500));
      __syncthreads();
    }
  }
}

}  // namespace hmg
