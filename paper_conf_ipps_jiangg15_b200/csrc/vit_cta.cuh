// vit_cta.cuh -- Viterbi filter (Alg 2 + Lazy-F) with one thread block per sequence.
//
// For long models (M up to 32*W*Q, e.g. 2048 with W = 16 warps x Q = 4 nodes) and for the
// latency-bound longest sequences, W warps cooperate on one DP row: thread g = 32*w + lane
// owns the contiguous nodes g*Q+1 .. g*Q+Q with its transition vectors and M/I/D cells in
// registers, as in vit_reg_kernel.  ONE block barrier per row:
//
//   D->D (Lazy-F, Fig 7) is resolved as a max-plus carry chain.  Each thread's
//   block of nodes maps an incoming D carry c to an outgoing max(cl, c + bsum), where cl is
//   the outgoing carry of its in-thread D chain (carry-in -inf) and bsum the sum of its tDD.  Inside a warp the incoming carries are found by shuffles
//   repeated while __any_sync reports a change (reading R19); across warps each warp
//   publishes its outgoing carry, and after the barrier every warp folds the carries of the
//   warps to its left itself (W <= 16 steps), so no further barrier round is needed.  With
//   sat(a + t) = max(a + t, -32768) and t <= 0 this is the same fixed point as the oracle's
//   sequential closure.
//   Diagonal carries across warp boundaries (row i-1 values at node 32*w*Q) are rebuilt by the
//   right-hand warp from the ingredients lane 31 of the left warp published before the barrier.
//   Hits (a row whose best M cell may move xB) are detected by the running-max vote of vit.cuh
//   folded into the same barrier (__syncthreads_or); only then is xE reduced over the block.
// Emission scores are s16 pairs; the 20 canonical rows and X live in shared memory (21 x M x 2 B:
// 86 KB at M = 2048, two blocks per SM), the rare codes (B J Z O U, gaps) are read from L2.
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
  static constexpr int SROWS = 21;           // shared rows: 20 canonical residues + X (code 26)
  static constexpr size_t table_bytes = (size_t)SROWS * ROWW * 4;
  // int scratch after the table
  static constexpr int XC = 0;               // [2][W][4]  lane 31: M, I, D (in-thread), carry into it
  static constexpr int WO = XC + 2 * W * 4;  // [2][W]     warp outgoing D carry (warp incoming = -inf)
  static constexpr int BW = WO + 2 * W;      // [W]        sum of tDD over the warp's nodes
  static constexpr int P31 = BW + W;         // [W]        lane 31: prefix of bsum inside the warp
  static constexpr int S31 = P31 + W;        // [W]        lane 31: prefix of tDD to its last node
  static constexpr int RX = S31 + W;         // [W]        per-warp xE max on hit rows
  static constexpr int PB = RX + W;          // [W+1]      exclusive prefix of BW over the warps
  static constexpr int NSCR = PB + W + 1;
};

template <int W, int Q>
__global__ void __launch_bounds__(32 * W, (W <= 8 ? 2 : 1)) vit_cta_kernel(const VitArgs a) {
  using S = VitCtaSmem<W, Q>;
  static_assert(Q % 2 == 0, "Q must be even (s16 emission pairs)");
  extern __shared__ uint4 smem4[];
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    constexpr int R16 = S::ROWW / 4;           // uint4 per row
    for (int i = threadIdx.x; i < 20 * R16; i += blockDim.x) smem4[i] = src[i];
    for (int i = threadIdx.x; i < R16; i += blockDim.x) smem4[20 * R16 + i] = src[26 * R16 + i];
  }
  uint32_t* tab = reinterpret_cast<uint32_t*>(smem4);
  int* scr = reinterpret_cast<int*>(reinterpret_cast<char*>(smem4) + S::table_bytes);
  __shared__ long long s_next;
  const int g = threadIdx.x;                 // DP lane
  const int w = g >> 5, lane = g & 31;

  // transitions of this thread's nodes (into-k BM MM IM DM, out-of-k MD MI II DD), s32
  // (B->M_k is re-read from global memory: it only matters when xB changes)
  int tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
  int ps[Q];
  const int32_t* tBMg = a.tr + g * Q;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = g * Q + q;
    const int NQ = S::NT * Q;
    tMM[q] = a.tr[1 * NQ + o]; tIM[q] = a.tr[2 * NQ + o]; tDM[q] = a.tr[3 * NQ + o];
    tMD[q] = a.tr[4 * NQ + o]; tMI[q] = a.tr[5 * NQ + o]; tII[q] = a.tr[6 * NQ + o]; tDD[q] = a.tr[7 * NQ + o];
  }
  int bsum = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    ps[q] = bsum;                            // sum of tDD before node q inside the thread
    bsum += tDD[q];
  }
  // exclusive prefix of bsum over the lanes of the warp (constant), and warp totals
  int pbs = bsum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, pbs, o);
    if (lane >= o) pbs += y;
  }
  pbs -= bsum;
  if (lane == 31) {
    scr[S::BW + w] = pbs + bsum;
    scr[S::P31 + w] = pbs;
    scr[S::S31 + w] = ps[Q - 1];
  }
  __syncthreads();
  if (g == 0) {
    int acc = 0;
    for (int v = 0; v < W; ++v) {
      scr[S::PB + v] = acc;
      acc += scr[S::BW + v];
    }
    scr[S::PB + W] = acc;
  }
  __syncthreads();
  // carry into warp w from warps v < w: PB[w] + max_v (WO[v] - PB[v+1]); lane v holds PB[v+1]
  const int pb_next = lane < W ? scr[S::PB + lane + 1] : 0;
  const int pb_w = scr[S::PB + w];
  const int pb_wl = w > 0 ? scr[S::PB + w - 1] : 0;
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
      Bk[q] = sadd(kBaseW + move, __ldg(tBMg + q));
    }
    int R = kNegW, xJ = kNegW;
    bool ovf = false;
    int thr = min(kBaseW + 501, 32767);
    // row -1 (all -inf) as seen from the right-hand warp
    int nbM = kNegW, nbI = kNegW, nbD = kNegW;
    int par = 0;
    uint32_t wcur = __ldcg(wp), wnxt = L > 6 ? __ldcg(wp + 1) : ~0u;
    for (int i = 0; i < L; ++i) {
      const int j6 = i % 6;
      const int x = (wcur >> (5 * j6)) & 31;
      if (j6 == 5) {                              // next word; prefetch the one after it
        wcur = wnxt;
        wnxt = (i / 6 + 2) * 6 < L ? __ldcg(wp + i / 6 + 2) : ~0u;
      }
      const uint32_t* rowp = x < 20 ? tab + x * S::ROWW
                                    : (x == 26 ? tab + 20 * S::ROWW
                                               : reinterpret_cast<const uint32_t*>(a.rsc) + x * S::ROWW);
      uint32_t e2[S::Q2];
      load_row<S::NT, S::Q2>(rowp, g, e2);
      int r[Q];
#pragma unroll
      for (int h = 0; h < S::Q2; ++h) {
        // s16 -> s32 on the FMA pipe (IMAD.HI), which this ALU-bound kernel leaves idle
        r[2 * h] = __mulhi((int)(e2[h] << 16), 65536);
        r[2 * h + 1] = __mulhi((int)e2[h], 65536);
      }
      // diagonal carries (row i-1 at node g*Q): lane l-1, or lane 31 of warp w-1 (nb*)
      int cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1);
      int cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1);
      int cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1);
      if (lane == 0) {
        cM = nbM;
        cI = nbI;
        cD = nbD;
      }
      // M and I (Alg 2 l.15-16, emission per reading R15)
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
      // D partial (l.17) + in-thread chain; this thread's outgoing carry is the chain's next link
      Dc[0] = kNegW;
#pragma unroll
      for (int q = 1; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], sadd(Mc[q - 1], tMD[q - 1]));
      const int cl = __viaddmax_s32(Dc[Q - 1], tDD[Q - 1], sadd(Mc[Q - 1], tMD[Q - 1]));
      // carries inside the warp: ci = outgoing of lane-1, iterate while any lane changes
      int out = cl, ci;
      for (;;) {
        ci = __shfl_up_sync(0xffffffffu, out, 1);
        if (lane == 0) ci = kNegW;
        const int o2 = max(cl, __viaddmax_s32(ci, bsum, kNegW));
        const bool chg = o2 != out;
        out = o2;
        if (!__any_sync(0xffffffffu, chg)) break;
      }
      const int wr = par * W + w;
      if (lane == 31) {
        scr[S::WO + wr] = out;                       // warp outgoing (warp incoming = -inf)
        scr[S::XC + wr * 4 + 0] = Mc[Q - 1];
        scr[S::XC + wr * 4 + 1] = Ic[Q - 1];
        scr[S::XC + wr * 4 + 2] = Dc[Q - 1];           // in-thread D of the last node (pre-carry)
        scr[S::XC + wr * 4 + 3] = ci;                  // intra-warp carry into lane 31
      }
      // the row's one barrier; hit / overflow vote folded in (reading R17)
      const bool hit = __syncthreads_or(R >= thr);
      // carries from the warps on the left: cw = into this warp, cwl = into warp w-1
      const int av = lane < W ? scr[S::WO + par * W + lane] - pb_next : kNegW * 64;
      const int m1 = __reduce_max_sync(0xffffffffu, lane < w ? av : kNegW * 64);
      const int m2 = __reduce_max_sync(0xffffffffu, lane + 1 < w ? av : kNegW * 64);
      const int cw = w > 0 ? max(kNegW, pb_w + m1) : kNegW;
      const int cwl = w > 1 ? max(kNegW, pb_wl + m2) : kNegW;
      const int cf = max(ci, __viaddmax_s32(cw, pbs, kNegW));    // final carry into this thread
      // apply the carry: D_q = max(D_q, cf + sum of the earlier tDD); runs die within a few
      // nodes, so walk two and finish only if some thread still improves
      {
        bool imp = cf > Dc[0];
        Dc[0] = max(Dc[0], cf);
        constexpr int K0 = Q <= 4 ? Q : 2;
#pragma unroll
        for (int q = 1; q < K0; ++q) {
          const int nd = __viaddmax_s32(Dc[q - 1], tDD[q - 1], kNegW);
          imp = imp && nd > Dc[q];
          Dc[q] = max(Dc[q], nd);
        }
        if constexpr (K0 < Q) {
          if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
            for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s32(Dc[q - 1], tDD[q - 1], Dc[q]);
          }
        }
      }
      // next row's diagonal carry for lane 0: warp w-1's last node, rebuilt here
      if (w > 0 && lane == 0) {
        const int* xc = scr + S::XC + (par * W + w - 1) * 4;
        const int cf31 = max(xc[3], __viaddmax_s32(cwl, scr[S::P31 + w - 1], kNegW));
        nbM = xc[0];
        nbI = xc[1];
        nbD = __viaddmax_s32(cf31, scr[S::S31 + w - 1], xc[2]);
      }
      if (hit) {
        int m = __reduce_max_sync(0xffffffffu, R);
        if (lane == 0) scr[S::RX + w] = m;
        __syncthreads();
        m = kNegW;
#pragma unroll
        for (int v = 0; v < W; ++v) m = max(m, scr[S::RX + v]);
        __syncthreads();
        if (!ovf) {
          if (m >= 32767) {
            ovf = true;
            thr = 0x7fffffff;
          } else {
            xJ = m - 500;
            const int xB = max(xJ, kBaseW) + move;
#pragma unroll
            for (int q = 0; q < Q; ++q) Bk[q] = sadd(xB, __ldg(tBMg + q));
            thr = min(max(xJ, kBaseW) + 501, 32767);
          }
        }
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
