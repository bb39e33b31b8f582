// vit_cpair.cuh -- Viterbi filter (Alg 2 + Lazy-F) for long models with one thread block per
// sequence and TWO cells per register (the s16x2 offset arithmetic of vit_pair.cuh in the block
// layout of vit_cta.cuh).
//
// NT = 32 W threads, 2 NT virtual lanes: virtual lane v owns nodes v Q + 1 .. v Q + Q; register
// q of thread g holds node g Q + q + 1 (low half) and node (g + NT) Q + q + 1 (high half).  The
// virtual warps are 0 .. W-1 (low halves of warps 0 .. W-1) then W .. 2W-1 (high halves).
//
// One block barrier per row (reading R19 / Fig 7 for Lazy-F):
//   * inside a warp, D->D carries move between lanes by shuffles repeated while __any_sync sees a
//     change (both halves at once: max(out, relu(c + bsum)) is one VIADDMNMX.RELU);
//   * across virtual warps the carry is a max-plus prefix in closed form,
//     c(vw) = max(0, PB[vw] + max_{v < vw} (WO[v] - PB[v+1])), PB = prefix of the warp tDD sums,
//     evaluated after the barrier from the published warp outputs WO (one REDUX per half);
//   * the diagonal carry into lane 0 (row i-1 at the last node of the previous virtual warp) is
//     rebuilt from what lane 31 of that warp published before the barrier.
// The floor F, the safe window and the re-basing on hit rows are those of VitPairLane; the whole
// block agrees on every special-state decision, so a sequence that leaves the window (re-score by
// the s32 kernel) or overflows stops at once.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"
#include "msv.cuh"        // load_row
#include "vit_pair.cuh"   // kRedo

namespace hmg {

template <int W, int Q, int SG = 1>
struct VitCPairSmem {
  static constexpr int NT = 32 * W;
  static constexpr int ROWW = Q * NT;          // s16x2 words per residue row
  static constexpr int SROWS = 21;             // 20 canonical residues + X (code 26) in shared memory
  static constexpr size_t table_bytes = (size_t)SROWS * ROWW * 4;
  // int scratch after the table
  // shared by the SG sequence groups of a block:
  static constexpr int PB = 0;                 // [2W+1] exclusive prefix of virtual-warp tDD sums
  static constexpr int P31 = PB + 2 * W + 1;   // [2W] lane 31: prefix of bsum inside its virtual warp
  static constexpr int S31 = P31 + 2 * W;      // [2W] lane 31: prefix of tDD up to its last node
  static constexpr int BW = S31 + 2 * W;       // [2W] virtual-warp tDD sums
  // per group (offset GRP * group index):
  static constexpr int G0 = (BW + 2 * W + 3) / 4 * 4;   // 16-byte aligned groups (uint4 XC)
  static constexpr int XC = 0;                 // [2][W][4] u32: lane 31 M, I, D (pre-carry), intra-warp carry
  static constexpr int WO = XC + 2 * W * 4;    // [2][W] u32: warp outgoing D carry (both halves)
  static constexpr int RX = WO + 2 * W;        // [W] u32 per-warp R max (hit rows)
  static constexpr int NX = (RX + W + 1) / 2 * 2;   // [2] next sequence index (long long)
  static constexpr int GRP = (NX + 2 + 3) / 4 * 4;
  static constexpr int NSCR = G0 + SG * GRP;
};

// named barrier of one sequence group (ids 1..SG; 0 is __syncthreads)
__device__ __forceinline__ void group_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ bool group_sync_or(int id, int nthreads, bool p) {
  int r;
  asm volatile(
      "{\n .reg .pred p, q;\n setp.ne.s32 p, %1, 0;\n barrier.red.or.pred q, %2, %3, p;\n selp.s32 %0, 1, 0, q;\n}"
      : "=r"(r)
      : "r"((int)p), "r"(id), "r"(nthreads)
      : "memory");
  return r != 0;
}

__device__ __forceinline__ int lo16(uint32_t v) { return (int)(int16_t)(v & 0xffffu); }
__device__ __forceinline__ int hi16(uint32_t v) { return (int)(int16_t)(v >> 16); }
__device__ __forceinline__ uint32_t pack16(int lo, int hi) {   // both in [0, 32767]
  return (uint32_t)lo | ((uint32_t)hi << 16);
}

template <int W, int Q, int SG>
__global__ void __launch_bounds__(32 * W * SG, 1) vit_cpair_kernel(const VitArgs a) {
  using S = VitCPairSmem<W, Q, SG>;
  constexpr int NT = S::NT;
  extern __shared__ uint4 smem4[];
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    constexpr int R16 = S::ROWW / 4;
    for (int i = threadIdx.x; i < 20 * R16; i += blockDim.x) smem4[i] = src[i];
    for (int i = threadIdx.x; i < R16; i += blockDim.x) smem4[20 * R16 + i] = src[26 * R16 + i];
  }
  const uint32_t* tab = reinterpret_cast<const uint32_t*>(smem4);
  int* scr = reinterpret_cast<int*>(reinterpret_cast<char*>(smem4) + S::table_bytes);
  const int grp = threadIdx.x / NT;                 // sequence group of this thread
  const int bid = 1 + grp;                          // its named barrier
  uint32_t* scru = reinterpret_cast<uint32_t*>(scr + S::G0 + grp * S::GRP);   // group scratch
  long long* s_next = reinterpret_cast<long long*>(scru + S::NX);
  const int g = threadIdx.x - grp * NT;             // DP lane inside the group
  const int w = g >> 5, lane = g & 31;
  const uint32_t* tr = reinterpret_cast<const uint32_t*>(a.tr);

  // transitions of this thread's nodes (s16x2, [8][NT][Q]); B->M re-read on hit rows
  uint32_t tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int o = g * Q + q;
    tMM[q] = tr[1 * NT * Q + o]; tIM[q] = tr[2 * NT * Q + o]; tDM[q] = tr[3 * NT * Q + o];
    tMD[q] = tr[4 * NT * Q + o]; tMI[q] = tr[5 * NT * Q + o]; tII[q] = tr[6 * NT * Q + o];
    tDD[q] = tr[7 * NT * Q + o];
  }
  // per half: sum of the thread's tDD (bsum), prefix up to its last node (s31), warp prefix (pbs)
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
    scr[S::BW + w] = pbs_lo + bs_lo;
    scr[S::BW + W + w] = pbs_hi + bs_hi;
    scr[S::P31 + w] = pbs_lo;
    scr[S::P31 + W + w] = pbs_hi;
    scr[S::S31 + w] = s31_lo;
    scr[S::S31 + W + w] = s31_hi;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int acc = 0;
    for (int v = 0; v < 2 * W; ++v) {
      scr[S::PB + v] = acc;
      acc += scr[S::BW + v];
    }
    scr[S::PB + 2 * W] = acc;
  }
  __syncthreads();
  // lane v (< 2W) holds PB[v+1] for the closed-form carry
  const int pb_next = lane < 2 * W ? scr[S::PB + lane + 1] : 0;
  const int pb_lo = scr[S::PB + w], pb_hi = scr[S::PB + W + w];
  // diagonal source of lane 0: low half <- virtual warp w-1 (none for w = 0),
  //                            high half <- virtual warp W+w-1 (w = 0: the low half of warp W-1)
  const int vs_lo = w - 1, vs_hi = W + w - 1;
  const int pbs_src_lo = vs_lo >= 0 ? scr[S::PB + vs_lo] : 0;
  const int pbs_src_hi = scr[S::PB + vs_hi];
  // D at the source's last node = max(D' published, relu(carry into the source warp + K))
  const int k_lo = vs_lo >= 0 ? scr[S::P31 + vs_lo] + scr[S::S31 + vs_lo] : 0;
  const int k_hi = scr[S::P31 + vs_hi] + scr[S::S31 + vs_hi];
  const int xsrc = w > 0 ? w - 1 : W - 1;         // warp whose lane 31 published the source values
  // prefix of tDD up to the thread's last node, per half (lane 31: D' = max(D, relu(ci + S31)))
  const uint32_t s31p = (uint32_t)(uint16_t)max(s31_lo, -32768) | ((uint32_t)(uint16_t)max(s31_hi, -32768) << 16);
  const long long ntot = a.list ? *a.nlist : a.nseq;
  const int safe = a.safe;
  constexpr int kNeg = -(1 << 30);

  for (;;) {
    if (g == 0) *s_next = (long long)atomicAdd(a.counter, 1ull);
    group_sync(bid, NT);
    const long long idx = *s_next;
    group_sync(bid, NT);
    if (idx >= ntot) break;
    const int s = a.list ? a.list[idx] : (int)idx;
    if (s < a.ndone && a.done[s]) continue;
    const int L = a.len[s];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    const int move = a.move[L];
    int F = max(-32768, kBaseW + move + a.tbm_min);
    int state = 0, xJ = kNegW;
    uint32_t Mc[Q], Ic[Q], Dc[Q], Bk[Q];
    bool okv = true;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      Mc[q] = Ic[q] = Dc[q] = 0u;                                   // Alg 2 l.9: -inf -> floor
      const uint32_t t = __ldg(tr + g * Q + q);
      const int lo = max(-32768, min(32767, kBaseW + move + lo16(t))) - F;
      const int hi = max(-32768, min(32767, kBaseW + move + hi16(t))) - F;
      okv = okv && lo <= safe && hi <= safe;
      Bk[q] = pack16(max(lo, 0), max(hi, 0));
    }
    if (group_sync_or(bid, NT, !okv)) state = 2;
    uint32_t R = 0u;
    int thr = min(min(kBaseW + 501, 32767) - F, safe + 1);         // in the offset domain
    uint32_t nbM = 0u, nbI = 0u, nbD = 0u;                        // lane 0: diagonal carries
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
      uint32_t e[Q];
      if (x < 20 || x == 26) {
        load_row<NT, Q>(tab + (x < 20 ? x : 20) * S::ROWW, g, e);     // shared memory
      } else {
        const uint32_t* rg = reinterpret_cast<const uint32_t*>(a.rsc) + x * S::ROWW;   // rare codes: L2
#pragma unroll
        for (int q = 0; q < Q; ++q) e[q] = 0u;
        load_row<NT, Q>(rg, g, e);
      }
      uint32_t cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1);
      uint32_t cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1);
      uint32_t cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1);
      if (lane == 0) {
        cM = nbM;
        cI = nbI;
        cD = nbD;
      }
#pragma unroll
      for (int q = Q - 1; q >= 0; --q) {
        const uint32_t pm = q ? Mc[q - 1] : cM;
        const uint32_t pi = q ? Ic[q - 1] : cI;
        const uint32_t pd = q ? Dc[q - 1] : cD;
        uint32_t m = __viaddmax_s16x2(pm, tMM[q], Bk[q]);
        m = __viaddmax_s16x2(pi, tIM[q], m);
        m = __viaddmax_s16x2(pd, tDM[q], m);
        Ic[q] = __viaddmax_s16x2(Ic[q], tII[q], __viaddmax_s16x2_relu(Mc[q], tMI[q], tMI[q]));
        Mc[q] = __viaddmax_s16x2_relu(m, e[q], e[q]);
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
      uint32_t out = cl, ci;
      for (;;) {
        ci = __shfl_up_sync(0xffffffffu, out, 1);
        if (lane == 0) ci = 0u;
        const uint32_t o2 = __viaddmax_s16x2_relu(ci, bsum2, cl);    // max(cl, relu(ci + bsum))
        const bool chg = o2 != out;
        out = o2;
        if (!__any_sync(0xffffffffu, chg)) break;
      }
      const int wr = par * W + w;
      if (lane == 31) {
        scru[S::WO + wr] = out;
        // the next row's diagonal source: M, I and D' = max(D, relu(ci + S31)), the last node's D
        // with the intra-warp carry applied (the cross-warp part is added by the reader)
        *reinterpret_cast<uint4*>(scru + S::XC + wr * 4) =
            make_uint4(Mc[Q - 1], Ic[Q - 1], __vmaxs2(Dc[Q - 1], __viaddmax_s16x2_relu(ci, s31p, s31p)), 0u);
      }
      const bool hit = ((__vadd2(R, (uint32_t)(0x8000 - thr) * 0x10001u) & 0x80008000u) != 0u);
      const bool anyhit = group_sync_or(bid, NT, hit);             // the row's one barrier
      // carries from the virtual warps on the left (closed form, both halves)
      const uint32_t wo = lane < W ? scru[S::WO + par * W + lane] : (lane < 2 * W ? scru[S::WO + par * W + lane - W] : 0u);
      const int av = lane < W ? lo16(wo) - pb_next : (lane < 2 * W ? hi16(wo) - pb_next : kNeg);
      const int m_lo = __reduce_max_sync(0xffffffffu, lane < w ? av : kNeg);
      const int m_hi = __reduce_max_sync(0xffffffffu, lane < W + w ? av : kNeg);
      const int cw_lo = w > 0 ? max(0, pb_lo + m_lo) : 0;
      const int cw_hi = max(0, pb_hi + m_hi);
      const uint32_t cf = __vmaxs2(ci, pack16(min(32767, max(0, cw_lo + pbs_lo)), min(32767, max(0, cw_hi + pbs_hi))));
      {
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
      // next row's diagonal carry for lane 0, from what the source warp's lane 31 published
      {
        const int m_slo = __reduce_max_sync(0xffffffffu, lane < vs_lo ? av : kNeg);
        const int m_shi = __reduce_max_sync(0xffffffffu, lane < vs_hi ? av : kNeg);
        const uint4 xc = *reinterpret_cast<const uint4*>(scru + S::XC + (par * W + xsrc) * 4);
        const int dl = vs_lo > 0 ? min(32767, max(0, pbs_src_lo + m_slo + k_lo)) : (vs_lo == 0 ? min(32767, max(0, k_lo)) : 0);
        const int dh = min(32767, max(0, max(0, pbs_src_hi + m_shi) + k_hi));
        if (w > 0) {
          nbM = xc.x;
          nbI = xc.y;
          nbD = __vmaxs2(xc.z, pack16(dl, dh));
        } else {                                   // low half: floor; high half <- warp W-1 low half
          nbM = __byte_perm(xc.x, 0u, 0x1054u);
          nbI = __byte_perm(xc.y, 0u, 0x1054u);
          nbD = __byte_perm(__vmaxs2(xc.z, pack16(dh, 0)), 0u, 0x1054u);
        }
      }
      if (anyhit) {                                                // Alg 2 l.22-24 on hit rows
        uint32_t mm = R;
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 16));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 8));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 4));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 2));
        mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 1));
        if (lane == 0) scru[S::RX + w] = mm;
        group_sync(bid, NT);
        int mp = 0;
#pragma unroll
        for (int v = 0; v < W; ++v) {
          const uint32_t t = scru[S::RX + v];
          mp = max(mp, max(lo16(t), hi16(t)));
        }
        group_sync(bid, NT);
        bool bad = false;
        if (mp > safe) {
          state = 2;                                   // beyond the 16-bit window: s32 re-score
        } else if (mp + F >= 32767) {
          state = 1;                                   // reading R17: overflow -> +inf, pass
        } else {
          xJ = mp + F - 500;                           // E->J (and E->C: xC == xJ)
          const int xB = max(xJ, kBaseW) + move;
          const int Fn = max(-32768, min(32767, xB + a.tbm_min));
          const int d = Fn - F;
          if (d > 0) {                                 // raise the floor: v' <- max(v' - d, 0)
            const uint32_t n = d >= 32768 ? 0x80008000u : (uint32_t)(uint16_t)(-d) * 0x10001u;
#pragma unroll
            for (int q = 0; q < Q; ++q) {
              Mc[q] = __viaddmax_s16x2_relu(Mc[q], n, n);
              Ic[q] = __viaddmax_s16x2_relu(Ic[q], n, n);
              Dc[q] = __viaddmax_s16x2_relu(Dc[q], n, n);
            }
            R = __viaddmax_s16x2_relu(R, n, n);
            nbM = __viaddmax_s16x2_relu(nbM, n, n);
            nbI = __viaddmax_s16x2_relu(nbI, n, n);
            nbD = __viaddmax_s16x2_relu(nbD, n, n);
          }
          F = Fn;
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            const uint32_t t = __ldg(tr + g * Q + q);
            const int lo = max(-32768, min(32767, xB + lo16(t))) - F;
            const int hi = max(-32768, min(32767, xB + hi16(t))) - F;
            bad = bad || lo > safe || hi > safe;
            Bk[q] = pack16(max(lo, 0), max(hi, 0));
          }
          thr = min(min(max(xJ, kBaseW) + 501, 32767) - F, safe + 1);
        }
        if (group_sync_or(bid, NT, bad)) state = 2;
      }
      par ^= 1;
      if (state) break;
     }
    }
    // final xC = max over rows of xE - 500
    uint32_t mm = R;
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 16));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 8));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 4));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 2));
    mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, 1));
    if (lane == 0) scru[S::RX + w] = mm;
    group_sync(bid, NT);
    if (g == 0) {
      int mp = 0;
      for (int v = 0; v < W; ++v) mp = max(mp, max(lo16(scru[S::RX + v]), hi16(scru[S::RX + v])));
      int raw;
      if (state == 1) raw = 32767;
      else if (state == 2) raw = kRedo;
      else if (mp > 0) raw = max(xJ, max(kNegW, mp + F - 500));
      else raw = xJ > kNegW ? xJ : kRedo;
      if (raw >= -32768) {
        a.raw_sorted[s] = (int16_t)raw;
      } else {
        const unsigned long long k = atomicAdd(a.redo_count, 1ull);
        a.redo_list[k] = s;
      }
    }
    group_sync(bid, NT);
  }
}

}  // namespace hmg
