// forward.cu -- Forward filter stage: the float Forward score of the survivors
// of the Viterbi filter, the stage after P7Viterbi in the hmmsearch pipeline (Fig 1 P:195-205:
// "Forward ... total log-likelihood ratios summed over all possible alignments").
//
// Model (readings F1-F5 in DESIGN.md): the same Plan-7 local multihit model the Viterbi
// filter scores, in probability (odds) space: M_k emits with odds exp(msc[k][x]), I/N/J/C emit
// with odds 1, transitions exp(tsc), local entry B->M_k = exp(tBM_k), exit M_k->E = D_k->E = 1,
// E->J = E->C = 1/2, length model N->N = J->J = C->C = L/(L+3), N->B = J->B = C->T = 3/(L+3).
// Row i (Alg 2's row order with sums in place of maxima):
//   M_k = (B tBM_k + M'_{k-1} tMM_k + I'_{k-1} tIM_k + D'_{k-1} tDM_k) e_k(x_i)
//   I_k = M'_k tMI_k + I'_k tII_k
//   D_{k+1} = M_k tMD_k + D_k tDD_k                      (the D->D chain, a linear recurrence)
//   E = sum_k (M_k + D_k);  N *= loop;  J = J loop + E/2;  C = C loop + E/2;  B = (N + J) move
// Score = log(C move) in nats.
//
// B200 design (fwd_kernel<W, Q>): a group of T = 32 W threads scores one sequence; thread t owns
// the contiguous node block t Q + 1 .. t Q + Q with the M/I/D cells and its 8 transition odds in
// registers (float32).  The D->D chain -- the part the paper resolves with Lazy-F passes in
// the max-plus filter -- is here a linear recurrence, so it is resolved EXACTLY in one pass by
// a scan of affine maps c -> a c + b (the sum-product analogue of the f1 max-plus scan,
// P:1279-1286): each thread folds its block into (a = prod tDD, b = chain from 0), a 5-step
// __shfl_up_sync scan composes the maps across the warp, one shared-memory step across warps,
// then each thread re-runs its block from its incoming carry.  Row values are kept in range by
// exact power-of-two rescaling (no rounding) whenever E exceeds 2^40, with the exponents
// accumulated in an integer.  Emission odds are staged in shared memory in a chunked layout
// (float4 per thread and chunk, conflict-free); rows that do not fit (long models) are read
// through L1 from the global copy of the table.  Sequences are taken from a length-sorted
// work queue (longest first) by whole groups.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <vector>

#include "hmg_internal.h"

namespace hmg {

constexpr float kFwdRescale = 1099511627776.0f;   // 2^40: E above this triggers a rescale


template <int Q> struct FwdVec { static constexpr int V = Q >= 4 ? 4 : Q; };

__device__ __forceinline__ void group_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

template <int W, int Q>
__global__ void __launch_bounds__(W * 32 > 256 ? W * 32 : 256, 1) fwd_kernel(const FwdArgs a) {
  constexpr int T = 32 * W;                    // threads per sequence
  constexpr int BT = T > 256 ? T : 256;        // threads per block
  constexpr int S = BT / T;                    // sequences per block
  constexpr int V = FwdVec<Q>::V;              // floats per vector load
  constexpr int C = Q / V;                     // chunks per thread
  constexpr int ROWF = T * Q;                  // floats per residue row
  extern __shared__ float4 smem4[];
  float* tab = reinterpret_cast<float*>(smem4);                   // [rows_smem][C][T][V]
  float* grp = tab + (size_t)a.rows_smem * ROWF;                   // per group scratch
  const int g = threadIdx.x / T, t = threadIdx.x % T, w = t >> 5, lane = t & 31;
  float2* agg = reinterpret_cast<float2*>(grp + g * (8 * W + 4));  // [W] warp affine aggregates
  float* epart = reinterpret_cast<float*>(agg + W);                // [W] warp partial sums of E
  float* cbuf = epart + W;                                         // [W][3] last node M, I, D
  int* slot = reinterpret_cast<int*>(cbuf + 3 * W);
  const int bar = 1 + g;

  // stage the emission odds (rows x < rows_smem) once per block
  {
    const float4* src = reinterpret_cast<const float4*>(a.etab);
    float4* dst = reinterpret_cast<float4*>(tab);
    const int n4 = a.rows_smem * ROWF / 4;
    for (int i = threadIdx.x; i < n4; i += BT) dst[i] = src[i];
  }
  // transition odds of this thread's nodes, and the thread's D->D map slope a = prod tDD
  float tBM[Q], tMM[Q], tIM[Q], tDM[Q], tMD[Q], tMI[Q], tII[Q], tDD[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const float* p = a.tr + (size_t)t * Q + q;
    tBM[q] = p[0 * T * Q]; tMM[q] = p[1 * T * Q]; tIM[q] = p[2 * T * Q]; tDM[q] = p[3 * T * Q];
    tMD[q] = p[4 * T * Q]; tMI[q] = p[5 * T * Q]; tII[q] = p[6 * T * Q]; tDD[q] = p[7 * T * Q];
  }
  float slope = 1.0f;
#pragma unroll
  for (int q = 0; q < Q; ++q) slope *= tDD[q];
  __syncthreads();

  const int64_t n = a.list ? *a.nlist : a.nseq;
  for (;;) {
    int64_t idx;
    if constexpr (W == 1) {
      unsigned long long v = 0;
      if (lane == 0) v = atomicAdd(a.counter, 1ull);
      idx = (int64_t)__shfl_sync(0xffffffffu, v, 0);
    } else {
      if (t == 0) *slot = (int)atomicAdd(a.counter, 1ull);
      group_sync(bar, T);
      idx = *slot;
      group_sync(bar, T);
    }
    if (idx >= n) break;
    const int s = a.list ? a.list[idx] : (int)idx;
    const int L = a.len[s];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    const float loop = (float)((double)L / (double)(L + 3));
    const float move = (float)(3.0 / (double)(L + 3));
    float Mc[Q], Ic[Q], Dc[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = 0.0f;
    float xN = 1.0f, xJ = 0.0f, xC = 0.0f, xB = move;
    int scale_exp = 0;                          // accumulated log2 of the rescalings
    bool row0 = true;                           // row 1: the diagonal carries are row 0's zeros
    float csc = 1.0f;                           // rescale applied after cbuf was written (row i-1)
    const int nw = (L + 5) / 6;
    for (int w0 = 0; w0 < nw; w0 += 32) {
      const uint32_t wreg = (w0 + lane < nw) ? __ldg(wp + w0 + lane) : 0u;
      const int wend = min(32, nw - w0);
#pragma unroll 1
      for (int j = 0; j < wend; ++j) {
        const uint32_t word = __shfl_sync(0xffffffffu, wreg, j);
        const int bend = min(6, L - 6 * (w0 + j));
#pragma unroll 1
        for (int b = 0; b < bend; ++b) {
          const int x = (word >> (5 * b)) & 31;
          // emission odds of the thread's nodes for residue x
          float e[Q];
          {
            const float* er = (x < a.rows_smem ? tab : a.etab) + (size_t)x * ROWF;
#pragma unroll
            for (int c = 0; c < C; ++c) {
              if constexpr (V == 4) {
                const float4 v = reinterpret_cast<const float4*>(er)[c * T + t];
                e[4 * c] = v.x; e[4 * c + 1] = v.y; e[4 * c + 2] = v.z; e[4 * c + 3] = v.w;
              } else if constexpr (V == 2) {
                const float2 v = reinterpret_cast<const float2*>(er)[c * T + t];
                e[2 * c] = v.x; e[2 * c + 1] = v.y;
              } else {
                e[c] = er[c * T + t];
              }
            }
          }
          // diagonal carries: row i-1 cells of node t Q (owned by thread t-1)
          float cM = __shfl_up_sync(0xffffffffu, Mc[Q - 1], 1);
          float cI = __shfl_up_sync(0xffffffffu, Ic[Q - 1], 1);
          float cD = __shfl_up_sync(0xffffffffu, Dc[Q - 1], 1);
          if (lane == 0) {
            if (W > 1 && w > 0 && !row0) {
              cM = cbuf[3 * (w - 1)] * csc; cI = cbuf[3 * (w - 1) + 1] * csc; cD = cbuf[3 * (w - 1) + 2] * csc;
            } else {
              cM = cI = cD = 0.0f;
            }
          }
          // M and I from row i-1 (descending q: Mc[q-1] still holds row i-1)
#pragma unroll
          for (int q = Q - 1; q >= 0; --q) {
            const float pm = q ? Mc[q - 1] : cM;
            const float pi = q ? Ic[q - 1] : cI;
            const float pd = q ? Dc[q - 1] : cD;
            float m = xB * tBM[q];
            m = fmaf(pm, tMM[q], m);
            m = fmaf(pi, tIM[q], m);
            m = fmaf(pd, tDM[q], m);
            Ic[q] = fmaf(Mc[q], tMI[q], Ic[q] * tII[q]);
            Mc[q] = m * e[q];
          }
          // D->D: the thread's affine map c -> slope c + b over its block, then the scan
          float bsum = 0.0f;
#pragma unroll
          for (int q = 0; q < Q; ++q) bsum = fmaf(Mc[q], tMD[q], bsum * tDD[q]);
          float ia = slope, ib = bsum;           // inclusive composite over lanes 0..lane
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const float ua = __shfl_up_sync(0xffffffffu, ia, d);
            const float ub = __shfl_up_sync(0xffffffffu, ib, d);
            if (lane >= d) {
              ib = fmaf(ia, ub, ib);
              ia *= ua;
            }
          }
          float cw = 0.0f;                       // D entering the warp's first node
          if constexpr (W > 1) {
            if (lane == 31) agg[w] = make_float2(ia, ib);
            group_sync(bar, T);
            for (int v = 0; v < w; ++v) {
              const float2 p = agg[v];
              cw = fmaf(p.x, cw, p.y);
            }
          }
          const float pa = __shfl_up_sync(0xffffffffu, ia, 1);
          const float pb = __shfl_up_sync(0xffffffffu, ib, 1);
          float dcur = lane == 0 ? cw : fmaf(pa, cw, pb);
          float esum = 0.0f;
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            Dc[q] = dcur;
            esum += Mc[q] + dcur;
            dcur = fmaf(Mc[q], tMD[q], dcur * tDD[q]);
          }
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) esum += __shfl_xor_sync(0xffffffffu, esum, o);
          float xE = esum;
          if constexpr (W > 1) {
            if (lane == 0) epart[w] = esum;
            if (lane == 31) {
              cbuf[3 * w] = Mc[Q - 1]; cbuf[3 * w + 1] = Ic[Q - 1]; cbuf[3 * w + 2] = Dc[Q - 1];
            }
            group_sync(bar, T);
            xE = 0.0f;
#pragma unroll
            for (int v = 0; v < W; ++v) xE += epart[v];
          }
          // specials (every thread, identical values)
          xN *= loop;
          xJ = fmaf(xJ, loop, 0.5f * xE);
          xC = fmaf(xC, loop, 0.5f * xE);
          csc = 1.0f;
          if (xE > kFwdRescale) {                // exact power-of-two rescale of the whole row
            const int ex = ilogbf(xE);
            const float sc = __int_as_float((127 - ex) << 23);
#pragma unroll
            for (int q = 0; q < Q; ++q) { Mc[q] *= sc; Ic[q] *= sc; Dc[q] *= sc; }
            xN *= sc; xJ *= sc; xC *= sc;
            csc = sc;                            // cbuf still holds the unscaled row
            scale_exp += ex;
          }
          xB = (xN + xJ) * move;
          row0 = false;
        }
      }
    }
    if (t == 0) {
      const double sc = (double)xC * (double)move;
      const int c = a.order[s];
      a.out[c] = sc > 0.0 ? (float)(log(sc) + (double)scale_exp * 0.6931471805599453) : -INFINITY;
      if (a.flags) a.flags[c] |= 8u;
    }
  }
}

using FwdFn = void (*)(const FwdArgs);

template <int W>
static FwdFn fwd_fn_q(int Q) {
  switch (Q) {
    case 2: return fwd_kernel<W, 2>;
    case 4: return fwd_kernel<W, 4>;
    case 8: return fwd_kernel<W, 8>;
  }
  return nullptr;
}

static FwdFn fwd_fn(int W, int Q) {
  switch (W) {
    case 1: return fwd_fn_q<1>(Q);
    case 2: return fwd_fn_q<2>(Q);
    case 4: return fwd_fn_q<4>(Q);
    case 8: return fwd_fn_q<8>(Q);
    case 16: return fwd_fn_q<16>(Q);
  }
  return nullptr;
}

static size_t fwd_group_floats(int W) { return (size_t)8 * W + 4; }

size_t fwd_smem(int W, int Q, int rows) {
  const int T = 32 * W, BT = std::max(T, 256), S = BT / T;
  return ((size_t)rows * T * Q + (size_t)S * fwd_group_floats(W)) * sizeof(float);
}

// Geometry: the fewest warps per sequence with 8 nodes per thread, then the fewest nodes per
// thread (2, 4, 8) for that width; models above 4096 nodes are not supported by this kernel.
bool fwd_geometry(int M, int* W, int* Q) {
  int w = 1;
  while (32 * w * 8 < M && w < 16) w *= 2;
  if (32 * w * 8 < M) return false;
  int q = 2;
  while (32 * w * q < M) q *= 2;
  *W = w;
  *Q = q;
  return true;
}

// Host tables (odds, float32) in the kernel's layouts.  msc: [M][29] nats, tsc: [M][8] nats.
void fwd_tables(int M, int W, int Q, const float* msc, const float* tsc, std::vector<float>* etab,
                std::vector<float>* tr) {
  const int T = 32 * W, V = Q >= 4 ? 4 : Q, C = Q / V, ROWF = T * Q;
  etab->assign((size_t)kRows * ROWF, 0.0f);
  for (int x = 0; x < kAlpha; ++x)
    for (int t = 0; t < T; ++t)
      for (int q = 0; q < Q; ++q) {
        const int k = t * Q + q;   // node k + 1
        if (k >= M) continue;
        const int c = q / V, v = q % V;
        (*etab)[(size_t)x * ROWF + ((size_t)c * T + t) * V + v] = expf(msc[(size_t)k * kAlpha + x]);
      }
  tr->assign((size_t)8 * T * Q, 0.0f);
  for (int s = 0; s < 8; ++s)
    for (int k = 0; k < M; ++k) (*tr)[(size_t)s * T * Q + k] = expf(tsc[(size_t)k * 8 + s]);
}

cudaError_t launch_fwd(int W, int Q, int rows_smem, const FwdArgs& a, cudaStream_t st, int* ok) {
  FwdFn fn = fwd_fn(W, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = fwd_smem(W, Q, rows_smem);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int BT = std::max(32 * W, 256);
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, BT, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) {
    *ok = 0;
    return cudaSuccess;
  }
  void* args[] = {const_cast<FwdArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel((const void*)fn, dim3((unsigned)(nsm * per)), dim3(BT), args, smem, st);
}

}  // namespace hmg
