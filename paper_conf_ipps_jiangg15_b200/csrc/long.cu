// long.cu -- the pipeline's long lane: whole-warp MSV then Viterbi for the longest sequences.
//
// A DP row cannot be split across time (Alg 1/2 carry xB from row i to i+1), so a
// sequence's filter time is bounded below by its length times the row latency of one
// lane group.  On a B200 the warp arbiter shares issue slots evenly among resident
// warps (measured: profiles/arbiter_r01.txt), so a long sequence sharing its SM
// sub-partition with five other warps runs five to six times slower than alone.
// The longest sequences (L > ~8x the mean) therefore run here: one warp per
// sequence, 4 warps per block, each block asking for enough shared memory to hold
// its SM alone, MSV with G = 32 (msv_batch<32, QL>) and -- if the MSV pass flag is
// set -- the Viterbi filter right away (VitLane<32, QV>).  The main MSV kernel runs
// concurrently on the remaining SMs; the Viterbi kernel later skips what ran here.
#include <cuda_runtime.h>

#include <algorithm>

#include "msv.cuh"
#include "vit.cuh"

namespace hmg {

// whole-warp MSV registers that cover a model of up to 32*QV nodes (2*32*QL >= 32*QV + 1)
__host__ __device__ constexpr int long_msv_q_of(int QV) { return (32 * QV + 1 + 63) / 64; }
int long_msv_q(int QV) { return long_msv_q_of(QV); }

template <int QV>
__global__ void __launch_bounds__(128) pipe_long_kernel(const LongArgs A) {
  constexpr int QL = long_msv_q_of(QV);
  constexpr int WM = kRows * QL * 32;       // MSV table words
  constexpr int WV = kRows * QV * 32;       // Viterbi emission table words
  extern __shared__ uint4 smem4[];
  {
    const uint4* s0 = reinterpret_cast<const uint4*>(A.m.prof);
    for (int i = threadIdx.x; i < WM / 4; i += blockDim.x) smem4[i] = s0[i];
    const uint4* s1 = reinterpret_cast<const uint4*>(A.v.rsc);
    for (int i = threadIdx.x; i < WV / 4; i += blockDim.x) smem4[WM / 4 + i] = s1[i];
  }
  __syncthreads();
  const uint32_t* smm = reinterpret_cast<const uint32_t*>(smem4);
  const int32_t* smv = reinterpret_cast<const int32_t*>(smem4) + WM;
  const int lane = threadIdx.x & 31;

  VitLane<32, QV> V;
#pragma unroll
  for (int q = 0; q < QV; ++q) {
    const int o = lane * QV + q;
    V.tBM[q] = A.v.tr[0 * 32 * QV + o];
    V.tMM[q] = A.v.tr[1 * 32 * QV + o];
    V.tIM[q] = A.v.tr[2 * 32 * QV + o];
    V.tDM[q] = A.v.tr[3 * 32 * QV + o];
    V.tMD[q] = A.v.tr[4 * 32 * QV + o];
    V.tMI[q] = A.v.tr[5 * 32 * QV + o];
    V.tII[q] = A.v.tr[6 * 32 * QV + o];
    V.tDD[q] = A.v.tr[7 * 32 * QV + o];
  }
  for (;;) {
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(A.counter, 1ull);
    b = __shfl_sync(0xffffffffu, b, 0);
    if ((long long)b >= A.nlong) break;
    const int s = (int)b;
    const int raw = msv_batch<32, QL>(A.m, smm, (long long)s, A.nlong);   // Alg 1
    const int L = A.m.len[s];
    const bool pass = raw == 255 || (raw != 254 && raw >= (int)A.thr[L]);
    if (!pass) continue;                      // 254: the exact MSV re-scores it; main stage decides
    // Alg 2 on this survivor, same warp, right away
    const uint32_t* wp = A.v.words + (size_t)A.v.woff16[s] * 4;
    const int nw = (L + 5) / 6;
    const int move = A.v.move[L];
#pragma unroll
    for (int q = 0; q < QV; ++q) V.Mc[q] = V.Ic[q] = V.Dc[q] = kNegW;
    int xB = kBaseW + move, xJ = kNegW, xC = kNegW;
    bool ovf = false;
    uint32_t wnext = __ldg(wp);
    for (int blk = 0; blk < nw; ++blk) {
      const uint32_t w = wnext;
      wnext = (blk + 1 < nw) ? __ldg(wp + blk + 1) : 0xffffffffu;
#pragma unroll
      for (int j = 0; j < 6; ++j) {
        const int x = (w >> (5 * j)) & 31;
        V.row(smv + x * (QV * 32), lane, xB, xJ, xC, move, ovf, x != kPadCode);
      }
    }
    if (lane == 0) {
      A.v.raw_sorted[s] = (int16_t)(ovf ? 32767 : xC);
      A.done[s] = 1;
    }
  }
}

namespace {
template <int QV>
const void* pick(int q) {
  if constexpr (QV > 16) {
    return nullptr;
  } else {
    if (q == QV) return reinterpret_cast<const void*>(&pipe_long_kernel<QV>);
    return pick<QV + 1>(q);
  }
}
}  // namespace

cudaError_t launch_pipe_long(int QV, const LongArgs& a, int nblocks, cudaStream_t st, int* ok) {
  const void* fn = pick<1>(QV);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  // ask for most of the SM's shared memory so no block of another kernel shares the SM
  const size_t need = ((size_t)kRows * long_msv_q_of(QV) * 32 + (size_t)kRows * QV * 32) * 4;
  int dev = 0, maxsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const size_t smem = std::max(need, (size_t)maxsm - 8192);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  void* args[] = {const_cast<LongArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)nblocks), dim3(128), args, smem, st);
}

}  // namespace hmg
