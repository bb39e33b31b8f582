// vit.cu -- Viterbi-filter launchers and the general (any M) kernel.
//
// vit_generic_kernel follows Alg 2 and Fig 7
// literally: one warp per sequence, lanes striding the model 32 nodes at a
// time (Alg 2 l.14), DP rows in global scratch, xE/Dmax by warp reduction, and
// the paper's parallel Lazy-F per 32-node window: every lane computes its DD
// candidate from its left neighbour, the window repeats while __any_sync finds
// a candidate that strictly improves a D cell (reading R19), then the last D
// carries into the next window (reading R20).  It serves models too long for
// the register kernel (vit_reg_kernel).
#include <cuda_runtime.h>

#include "vit.cuh"

namespace hmg {

const void* vit_reg_ptr_g8(int q);
const void* vit_reg_ptr_g16(int q);
const void* vit_reg_ptr_g32(int q);

int vit_q_max(int G) { return 16; }

static const void* vit_reg_ptr(int G, int Q) {
  switch (G) {
    case 8: return vit_reg_ptr_g8(Q);
    case 16: return vit_reg_ptr_g16(Q);
    case 32: return vit_reg_ptr_g32(Q);
  }
  return nullptr;
}

cudaError_t launch_vit_reg(int G, int Q, const VitArgs& a, cudaStream_t st, int* ok) {
  const void* fn = vit_reg_ptr(G, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = (((size_t)kRows * Q * G + 3) / 4) * 16;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 128, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  int64_t grid = (int64_t)nsm * per;
  void* args[] = {const_cast<VitArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(128), args, smem, st);
}

__global__ void __launch_bounds__(256) vit_generic_kernel(const VitArgs a) {
  const int lane = threadIdx.x & 31;
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  const int M = a.M;
  int* Mp = a.scratch + (size_t)warp * 6 * (M + 1);
  int* Ip = Mp + (M + 1);
  int* Dp = Ip + (M + 1);
  int* Mn = Dp + (M + 1);
  int* In = Mn + (M + 1);
  int* Dn = In + (M + 1);
  const int32_t* tBM = a.tr + 0 * (size_t)M; const int32_t* tMM = a.tr + 1 * (size_t)M;
  const int32_t* tIM = a.tr + 2 * (size_t)M; const int32_t* tDM = a.tr + 3 * (size_t)M;
  const int32_t* tMD = a.tr + 4 * (size_t)M; const int32_t* tMI = a.tr + 5 * (size_t)M;
  const int32_t* tII = a.tr + 6 * (size_t)M; const int32_t* tDD = a.tr + 7 * (size_t)M;
  const long long n = a.list ? *a.nlist : a.nseq;
  for (long long idx = warp; idx < n; idx += nwarps) {
    const int s = a.list ? a.list[idx] : (int)idx;
    const int L = a.len[s];
    const int move = a.move[L];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    for (int k = lane; k <= M; k += 32) Mp[k] = Ip[k] = Dp[k] = kNegW;     // l.9
    if (lane == 0) Mn[0] = In[0] = Dn[0] = kNegW;
    __syncwarp();
    const int xN = kBaseW;
    int xB = xN + move, xJ = kNegW, xC = kNegW;
    bool ovf = false;
    for (int i = 0; i < L; ++i) {                                          // l.10
      const int x = (__ldg(wp + i / 6) >> (5 * (i % 6))) & 31;            // l.11
      const int16_t* r = a.rsc + (size_t)x * M;
      int xE = kNegW;                                                      // l.12
      for (int k = 1 + lane; k <= M; k += 32) {                           // l.14
        int m = sadd(xB, tBM[k - 1]);                                      // l.16 (+ R15)
        m = max(m, sadd(Mp[k - 1], tMM[k - 1]));
        m = max(m, sadd(Ip[k - 1], tIM[k - 1]));
        m = max(m, sadd(Dp[k - 1], tDM[k - 1]));
        m = sadd(m, (int)__ldg(r + k - 1));
        Mn[k] = m;
        In[k] = max(sadd(Mp[k], tMI[k - 1]), sadd(Ip[k], tII[k - 1]));  // l.15
        xE = max(xE, m);                                                   // l.18
      }
      xE = __reduce_max_sync(0xffffffffu, xE);                             // l.22
      __syncwarp();
      if (xE >= 32767) { ovf = true; break; }
      xC = max(xC, xE - 500);                                              // l.24
      xJ = max(xJ, xE - 500);
      xB = max(xJ, xN) + move;
      // l.17 partial D + l.25 parallel Lazy-F by 32-node windows (Fig 7)
      int carry = kNegW;   // DD candidate entering the window from node k0-1
      for (int k0 = 1; k0 <= M; k0 += 32) {
        const int k = k0 + lane;
        const bool in = k <= M;
        int d = (in && k >= 2) ? sadd(Mn[k - 1], tMD[k - 2]) : kNegW;
        const int tdd = (in && k >= 2) ? tDD[k - 2] : kNegW;   // D_{k-1} -> D_k
        for (;;) {
          const int left = __shfl_up_sync(0xffffffffu, d, 1);
          const int cand = (lane == 0) ? carry : sadd(left, tdd);
          const bool imp = in && cand > d;
          if (!__any_sync(0xffffffffu, imp)) break;
          if (imp) d = cand;
        }
        if (in) Dn[k] = d;
        const int last = __shfl_sync(0xffffffffu, d, 31);
        const int knext = k0 + 32;                            // first node of next window
        carry = (knext <= M) ? sadd(last, tDD[knext - 2]) : kNegW;
      }
      __syncwarp();
      int* t;
      t = Mp; Mp = Mn; Mn = t;
      t = Ip; Ip = In; In = t;
      t = Dp; Dp = Dn; Dn = t;
    }
    if (lane == 0) a.raw_sorted[s] = (int16_t)(ovf ? 32767 : xC);         // l.28
    __syncwarp();
  }
}

cudaError_t launch_vit_generic(const VitArgs& a, int nwarps, cudaStream_t st) {
  const int threads = 256;
  const int blocks = (nwarps * 32 + threads - 1) / threads;
  g_launches += 1;
  vit_generic_kernel<<<blocks, threads, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace hmg
