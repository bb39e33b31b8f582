// forward.cuh -- the Forward-stage kernel fwd_kernel<W, Q, S> (see forward.cu for the model,
// the design and the host side).  W warps score one sequence, each thread owns Q contiguous
// nodes, a block holds S sequences sharing one shared-memory copy of the emission odds.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"

namespace hmg {

constexpr float kFwdRescale = 1099511627776.0f;   // 2^40: E above this triggers a rescale


// floats per vector load of the emission row: 4 when Q is a multiple of 4, else 2, else 1 (the
// one-warp geometries with 12..14 nodes per thread fit M = 385..448 without 16-node padding)
template <int Q> struct FwdVec { static constexpr int V = Q % 4 == 0 ? 4 : (Q % 2 == 0 ? 2 : 1); };

__device__ __forceinline__ void group_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Per-thread scan constants (host-computed from tDD, fwd_tables): the D->D carry into thread t is
// c_in(t) = sum_{j<t} b_j prod_{j<m<t} a_m with a_m = prod of thread m's tDD and b_j its chain
// from zero, so every slope in the scan is a profile constant and only the b's move per row.
//   0..4  mul_d   slope of lanes (t-d, t] for the Hillis-Steele step d = 1, 2, 4, 8, 16
//   5     pa      slope of lanes [warp start, t)        6  ai  slope of lanes [warp start, t]
//   7     G       sum_{t'>t} Psum(t') prod_{t<m<t'} a_m  (E = sum_t [sum_q (M + Dloc) + b_t G_t])
//   8     pa P_{Q-1}
//   9..   P_q     prod_{q'<q} tDD_{q'} within the thread (D_q = Dloc_q + c_in P_q)
constexpr int kFwdConst = 9;

// GL < 32 (W = 1 only): a sequence takes a group of GL lanes and a warp scores 32 / GL sequences of
// adjacent length rank in lockstep, iterating to the longest of them (rows past a sequence's end
// leave its special states untouched); shuffles run within the GL-lane segments.
template <int W, int Q, int S, int GL = 32>
__global__ void __launch_bounds__((W == 1 ? GL : 32 * W) * S, 1) fwd_kernel(const FwdArgs a) {
  static_assert(GL == 32 || W == 1, "lane groups below a warp need W = 1");
  constexpr int T = W == 1 ? GL : 32 * W;      // threads per sequence
  constexpr int BT = T * S;                    // threads per block (S sequences)
  constexpr int NGW = 32 / T > 0 ? 32 / T : 1; // sequences per warp
  constexpr int LG = GL == 8 ? 3 : GL == 16 ? 4 : 5;   // scan / reduction steps
  constexpr int V = FwdVec<Q>::V;              // floats per vector load
  constexpr int C = Q / V;                     // chunks per thread
  constexpr int ROWF = T * Q;                  // floats per residue row
  constexpr int PAR = (7 * W + 3) / 4 * 4;     // floats per parity buffer of a group (16-B aligned)
  extern __shared__ float4 smem4[];
  float* tab = reinterpret_cast<float*>(smem4);                   // [rows_smem][C][T][V]
  const int g = threadIdx.x / T, t = threadIdx.x % T, w = t >> 5, lane = t & (GL - 1);
  float* grp = tab + (size_t)a.rows_smem * ROWF + (size_t)g * (2 * PAR + 4);
  int* slot = reinterpret_cast<int*>(grp + 2 * PAR);
  const int bar = 1 + g;

  {  // stage the emission odds (rows x < rows_smem) once per block
    const float4* src = reinterpret_cast<const float4*>(a.etab);
    float4* dst = reinterpret_cast<float4*>(tab);
    const int n4 = a.rows_smem * ROWF / 4;
    for (int i = threadIdx.x; i < n4; i += BT) dst[i] = src[i];
  }
  // LEAN (Q = 16): no per-node P registers; D = Dloc + c_in P is applied as two 8-node product
  // chains (c_in and c_in P_8), keeping the thread at ~220 registers so one warp holds 512 nodes
  constexpr bool LEAN = Q >= 16;
  constexpr int NP = LEAN ? 1 : Q;
  float tBM[Q], tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q], P[NP];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const float* p = a.tr + (size_t)t * Q + q;
    tBM[q] = p[0 * T * Q]; tMM[q] = p[1 * T * Q]; tIM[q] = p[2 * T * Q]; tDM[q] = p[3 * T * Q];
    tMD[q] = p[4 * T * Q]; tMI[q] = p[5 * T * Q]; tII[q] = p[6 * T * Q]; tDD[q] = p[7 * T * Q];
    if constexpr (!LEAN) P[q] = a.cst[(kFwdConst + q) * T + t];
  }
  if constexpr (LEAN) P[0] = a.cst[(kFwdConst + Q / 2) * T + t];   // P_{Q/2}
  const float PL = a.cst[(kFwdConst + Q - 1) * T + t];             // P_{Q-1} (cross-warp carry)
  float mul[LG];
#pragma unroll
  for (int d = 0; d < LG; ++d) mul[d] = a.cst[d * T + t];
  const float pa = a.cst[5 * T + t], ai = a.cst[6 * T + t], G = a.cst[7 * T + t], paP = a.cst[8 * T + t];
  __syncthreads();

  const int64_t n = a.list ? *a.nlist : a.nseq;
  int par = 0;
  for (;;) {
    int64_t idx;
    if constexpr (W == 1) {                    // one fetch per warp: NGW adjacent sequences
      unsigned long long v = 0;
      if ((threadIdx.x & 31) == 0) v = atomicAdd(a.counter, (unsigned long long)NGW);
      idx = (int64_t)__shfl_sync(0xffffffffu, v, 0);
      if (idx >= n) break;
      idx += (threadIdx.x & 31) / T;
    } else {
      if (t == 0) *slot = (int)atomicAdd(a.counter, 1ull);
      group_sync(bar, T);
      idx = *slot;
      group_sync(bar, T);
      if (idx >= n) break;
    }
    const bool valid = idx < n;
    const int s = valid ? (a.list ? a.list[idx] : (int)idx) : 0;
    const int L = valid ? a.len[s] : 0;
    int Lw = L;                                // rows the warp iterates: its longest sequence
#pragma unroll
    for (int o = 16; o >= T; o >>= 1) Lw = max(Lw, __shfl_xor_sync(0xffffffffu, Lw, o));
    const uint32_t* wp = a.words + (size_t)(valid ? a.woff16[s] : 0) * 4;
    const float loop = valid ? (float)((double)L / (double)(L + 3)) : 0.0f;
    const float move = valid ? (float)(3.0 / (double)(L + 3)) : 0.0f;
    float Mc[Q], Ic[Q], Dc[Q], e[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = 0.0f;
    float nM = 0.0f, nI = 0.0f, nD = 0.0f;     // lane 0 of warp w > 0: row i-1 cells of node t Q
    float xN = 1.0f, xJ = 0.0f, xC = 0.0f, xB = move;
    int scale_exp = 0;                          // accumulated log2 of the rescalings
    auto load_row = [&](const float* er, bool shared) {
#pragma unroll
      for (int c = 0; c < C; ++c) {
        if constexpr (V == 4) {
          const float4* p4 = reinterpret_cast<const float4*>(er) + c * T + t;
          const float4 v = shared ? *p4 : __ldg(p4);
          e[4 * c] = v.x; e[4 * c + 1] = v.y; e[4 * c + 2] = v.z; e[4 * c + 3] = v.w;
        } else if constexpr (V == 2) {
          const float2* p2 = reinterpret_cast<const float2*>(er) + c * T + t;
          const float2 v = shared ? *p2 : __ldg(p2);
          e[2 * c] = v.x; e[2 * c + 1] = v.y;
        } else {
          const float* p1 = er + c * T + t;
          e[c] = shared ? *p1 : __ldg(p1);
        }
      }
    };
    const int nw = (L + 5) / 6, nww = (Lw + 5) / 6;
    for (int w0 = 0; w0 < nww; w0 += GL) {
      const uint32_t wreg = (w0 + lane < nw) ? __ldcg(wp + w0 + lane) : 0u;
      const int wend = min(GL, nww - w0);
#pragma unroll 1
      for (int j = 0; j < wend; ++j) {
        const uint32_t word = __shfl_sync(0xffffffffu, wreg, j, GL);
        const int bend = min(6, Lw - 6 * (w0 + j));
#pragma unroll 1
        for (int b = 0; b < bend; ++b) {
          // rows past the sequence's end (lane groups only): cells only, specials frozen
          const bool act = T >= 32 || 6 * (w0 + j) + b < L;
          const int x = act ? (int)((word >> (5 * b)) & 31) : 0;
          // x is uniform over the group (>= one warp): shared-memory rows by LDS, the rest via L1
          if (x < a.rows_smem) load_row(tab + (size_t)x * ROWF, true);
          else load_row(a.etab + (size_t)x * ROWF, false);
          // diagonal carries: row i-1 cells of node t Q (thread t-1)
          float cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1, GL);
          float cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1, GL);
          float cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1, GL);
          if (lane == 0) { cM = nM; cI = nI; cD = nD; }
          // M and I from row i-1 (descending q: index q-1 still holds row i-1)
#pragma unroll
          for (int q = Q - 1; q >= 0; --q) {
            const float pm = q ? Mc[q - 1] : cM;
            const float pi = q ? Ic[q - 1] : cI;
            const float pd = q ? Dc[q - 1] : cD;
            float m = pm * tMM[q];
            m = fmaf(pi, tIM[q], m);
            m = fmaf(pd, tDM[q], m);
            m = fmaf(xB, tBM[q], m);
            Ic[q] = fmaf(Mc[q], tMI[q], Ic[q] * tII[q]);
            Mc[q] = m * e[q];
          }
          // D->D within the thread from a zero carry (Dloc), the thread's contribution to E
          float bsum = 0.0f, econ = 0.0f;
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            Dc[q] = bsum;
            econ += Mc[q] + bsum;
            bsum = fmaf(bsum, tDD[q], Mc[q] * tMD[q]);
          }
          econ = fmaf(bsum, G, econ);
          // scan of the chain outputs (constant slopes) and the E reduction, independent chains
          float ib = bsum;
#pragma unroll
          for (int d = 0; d < LG; ++d) {
            const float ub = __shfl_up_sync(0xffffffffu, ib, 1 << d, GL);
            econ += __shfl_xor_sync(0xffffffffu, econ, (GL / 2) >> d);
            if (lane >= (1 << d)) ib = fmaf(mul[d], ub, ib);
          }
          const float pb = __shfl_up_sync(0xffffffffu, ib, 1, GL);
          float xE = econ, cw = 0.0f;
          if constexpr (W > 1) {
            float* buf = grp + par * PAR;
            float4* cbuf = reinterpret_cast<float4*>(buf);           // [W] last node M, I, D decomposition
            float2* agg = reinterpret_cast<float2*>(buf + 4 * W);    // [W] (slope, b) of each warp
            float* epart = buf + 6 * W;                              // [W]
            if (lane == 31) {
              agg[w] = make_float2(ai, ib);
              cbuf[w] = make_float4(Mc[Q - 1], Ic[Q - 1], fmaf(pb, PL, Dc[Q - 1]), paP);
            }
            if (lane == 0) epart[w] = econ;
            group_sync(bar, T);
            xE = 0.0f;
#pragma unroll
            for (int v = 0; v < W; ++v) xE += epart[v];
            float cprev = 0.0f;
            for (int v = 0; v < w; ++v) {
              cprev = cw;
              const float2 pv = agg[v];
              cw = fmaf(pv.x, cw, pv.y);
            }
            if (lane == 0 && w > 0) {
              const float4 c = cbuf[w - 1];
              nM = c.x; nI = c.y; nD = fmaf(c.w, cprev, c.z);
            }
            par ^= 1;
          }
          // row i's D: Dloc + c_in P
          const float cin = lane == 0 ? cw : fmaf(pa, cw, pb);
          if constexpr (LEAN) {
            float c0 = cin, c1 = cin * P[0];
#pragma unroll
            for (int q = 0; q < Q / 2; ++q) {
              Dc[q] += c0;
              Dc[q + Q / 2] += c1;
              c0 *= tDD[q];
              c1 *= tDD[q + Q / 2];
            }
          } else {
#pragma unroll
            for (int q = 0; q < Q; ++q) Dc[q] = fmaf(cin, P[q], Dc[q]);
          }
          // specials (every thread of the group, identical values; frozen past the sequence's end)
          if (T < 32 && !act) continue;
          xN *= loop;
          xJ = fmaf(xJ, loop, 0.5f * xE);
          xC = fmaf(xC, loop, 0.5f * xE);
          if (xE > kFwdRescale) {                // exact power-of-two rescale of the whole row
            const int ex = ilogbf(xE);
            const float sc = __int_as_float((127 - ex) << 23);
#pragma unroll
            for (int q = 0; q < Q; ++q) { Mc[q] *= sc; Ic[q] *= sc; Dc[q] *= sc; }
            nM *= sc; nI *= sc; nD *= sc;
            xN *= sc; xJ *= sc; xC *= sc;
            scale_exp += ex;
          }
          xB = (xN + xJ) * move;
        }
      }
    }
    if (t == 0 && valid) {
      const double sc = (double)xC * (double)move;
      const int c = a.order[s];
      a.out[c] = sc > 0.0 ? (float)(log(sc) + (double)scale_exp * 0.6931471805599453) : -INFINITY;
      if (a.flags) a.flags[c] |= 8u;
    }
  }
}

}  // namespace hmg
