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

#include "forward.cuh"

namespace hmg {

const void* fwd_ptr_w1(int q, int s);
const void* fwd_ptr_w2(int q, int s);
const void* fwd_ptr_w4(int q, int s);
const void* fwd_ptr_w8(int q, int s);
const void* fwd_ptr_w16(int q, int s);
const void* fwd_ptr_sub(int gl, int q, int s);

// T = threads per sequence: 8 (sub-warp lane groups) or 32 W.
static const void* fwd_fn(int T, int Q, int S) {
  switch (T) {
    case 8: return fwd_ptr_sub(T, Q, S);
    case 32: return fwd_ptr_w1(Q, S);
    case 64: return fwd_ptr_w2(Q, S);
    case 128: return fwd_ptr_w4(Q, S);
    case 256: return fwd_ptr_w8(Q, S);
    case 512: return fwd_ptr_w16(Q, S);
  }
  return nullptr;
}

static const int* fwd_s_list(int T) {
  static const int s8[] = {8, 16, 32, 0}, s32[] = {2, 4, 8, 12, 0}, s64[] = {1, 2, 4, 6, 0},
                   s128[] = {1, 2, 3, 0}, s256[] = {1, 0};
  switch (T) {
    case 8: return s8;
    case 32: return s32;
    case 64: return s64;
    case 128: return s128;
  }
  return s256;
}

static size_t fwd_group_floats(int T) {        // forward.cuh: 2 parity buffers + slot
  const int W = T >= 32 ? T / 32 : 1;
  return (size_t)2 * ((7 * W + 3) / 4 * 4) + 4;
}

size_t fwd_smem(int T, int Q, int rows, int S) {
  return ((size_t)rows * T * Q + (size_t)S * fwd_group_floats(T)) * sizeof(float);
}

// Sequences per block: the instantiated S with the most resident warps per SM (registers and the
// shared emission table decide), the smaller S on ties (finer work granularity).
int fwd_pick_s(int T, int Q, int rows) {
  int best = 0, bw = 0;
  for (const int* ps = fwd_s_list(T); *ps; ++ps) {
    const int S = *ps;
    const void* fn = fwd_fn(T, Q, S);
    if (!fn) continue;
    const size_t smem = fwd_smem(T, Q, rows, S);
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) {
      cudaGetLastError();
      continue;
    }
    int per = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, T * S, smem) != cudaSuccess) {
      cudaGetLastError();
      continue;
    }
    const int warps = per * T * S / 32;
    if (warps > bw) {
      bw = warps;
      best = S;
    }
  }
  return best;
}

// Geometry (T threads per sequence, Q nodes per thread): models up to 32 nodes take sub-warp
// groups of 8 lanes (4 sequences per warp, SURVEY 7 hard part 5: at M = 64-128 the 8/16-lane
// groups with 8 nodes per thread measured 10% slower than a warp with 2-4 nodes, whose lower
// register count doubles the resident warps); above,
// the fewest warps at qmax nodes per thread (16 for the lean variant, up to 8 warps; else 8, up
// to 16 warps), then the fewest nodes per thread for that width; above 4096 nodes: none.
bool fwd_geometry(int M, int* T, int* Q, int qmax) {
  if (M <= 32) {                       // measured: only tiny models gain (profiles/fwd_bench_r01f.jsonl)
    *T = 8;
    *Q = M <= 16 ? 2 : 4;
    return true;
  }
  const int wmax = qmax >= 16 ? 8 : 16;   // 16 nodes/thread: <= 256 threads per sequence (registers)
  int w = 1;
  while (32 * w * qmax < M && w < wmax) w *= 2;
  if (32 * w * qmax < M) return false;
  int q = 2;
  while (32 * w * q < M) q *= 2;
  // one warp: 12 / 13 / 14 nodes per thread where they fit below 16 (M = 257 ... 448: at M = 400,
  // 13 nodes -- 416 cells a row -- instead of 512)
#ifndef FWD_NO_Q13
  if (w == 1 && q == 16 && qmax >= 16)
#else
  if (false)                                      // A/B builds: powers of two only
#endif
    for (int qq = 12; qq < 16; ++qq)
      if (qq != 15 && 32 * qq >= M) {
        q = qq;
        break;
      }
  *T = 32 * w;
  *Q = q;
  return true;
}

// Host tables (odds, float32) in the kernel's layouts.  msc: [M][29] nats, tsc: [M][8] nats.
void fwd_tables(int M, int T, int Q, const float* msc, const float* tsc, std::vector<float>* etab,
                std::vector<float>* tr, std::vector<float>* cst) {
  const int V = Q % 4 == 0 ? 4 : (Q % 2 == 0 ? 2 : 1);   // FwdVec<Q>::V (forward.cuh)
  const int C = Q / V, ROWF = T * Q, SEG = T < 32 ? T : 32;   // SEG: shuffle segment
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
  // scan constants (kernel comment), from the float odds the kernel uses, in double
  std::vector<double> A(T), Pd((size_t)T * Q), Ps(T);
  for (int t = 0; t < T; ++t) {
    double p = 1.0, ps = 0.0;
    for (int q = 0; q < Q; ++q) {
      Pd[(size_t)t * Q + q] = p;
      ps += p;
      p *= (double)(*tr)[(size_t)7 * T * Q + t * Q + q];
    }
    A[t] = p;
    Ps[t] = ps;
  }
  auto slope = [&](int lo, int hi) {   // prod A[lo..hi], 1 if empty
    double r = 1.0;
    for (int m = lo; m <= hi; ++m) r *= A[m];
    return r;
  };
  cst->assign((size_t)(kFwdConst + Q) * T, 0.0f);
  auto C_ = [&](int i, int t) -> float& { return (*cst)[(size_t)i * T + t]; };
  for (int t = 0; t < T; ++t) {
    const int ws = t & ~(SEG - 1), lane = t & (SEG - 1);
    for (int d = 0; d < 5; ++d)
      C_(d, t) = (1 << d) < SEG && lane >= (1 << d) ? (float)slope(t - (1 << d) + 1, t) : 0.0f;
    C_(5, t) = (float)slope(ws, t - 1);
    C_(6, t) = (float)slope(ws, t);
    double g = 0.0, run = 1.0;          // G_t = sum_{t'>t} Ps(t') prod_{t<m<t'} A_m
    for (int u = t + 1; u < T; ++u) {   // (over the whole sequence's threads)
      g += Ps[u] * run;
      run *= A[u];
    }
    C_(7, t) = (float)g;
    C_(8, t) = (float)(slope(ws, t - 1) * Pd[(size_t)t * Q + Q - 1]);
    for (int q = 0; q < Q; ++q) C_(kFwdConst + q, t) = (float)Pd[(size_t)t * Q + q];
  }
}

cudaError_t launch_fwd(int T, int Q, int S, int rows_smem, const FwdArgs& a, cudaStream_t st, int* ok) {
  const void* fn = fwd_fn(T, Q, S);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = fwd_smem(T, Q, rows_smem, S);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int BT = T * S;
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
  return cudaLaunchKernel(fn, dim3((unsigned)(nsm * per)), dim3(BT), args, smem, st);
}

}  // namespace hmg
