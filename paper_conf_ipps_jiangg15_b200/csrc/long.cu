// long.cu -- the long-sequence lane (sequences with L > ~8x the mean length).
//
// A DP row cannot be split across time (Alg 1/2 carry xB from row i to i+1), so a
// sequence's filter time is bounded below by its length times the row latency of one
// lane group; and the B200 warp arbiter shares issue slots evenly among resident warps
// (measured, profiles/arbiter_r01.txt), so a long sequence sharing its SM sub-partition
// with five other warps runs five to six times slower than alone.
//
// MSV of a long sequence is cut into row chunks that run in parallel, each from the empty
// state M rows early.  Exact while xB is unchanged: an MSV domain is one ungapped diagonal,
// so row i depends only on rows > i - M.  The last chunk of a sequence to finish combines
// the chunk maxima; if any chunk saw a row that could move xB (a hit) or overflow, it
// re-runs the sequence with the sequential whole-warp DP (msv_batch<32, QL>).
//   pipe_long_msv_kernel<QL>   chunked MSV only (hmg_msv), on the whole GPU before the main
//                              MSV kernel;
//   pipe_long_vit_kernel<QV>   the Viterbi filter (latency variant of VitLane) of the long
//                              sequences that pass, on SMs it holds alone, while the main MSV
//                              kernel (programmatic dependent launch) fills the other SMs
//                              (hmg_pipeline);
//   pipe_long_vpair_kernel<Q>  the same with the s16x2 pair lane (vit_pair.cuh), whole warp,
//                              for models up to 1024 nodes; sequences it cannot score in its
//                              16-bit window are left to the main Viterbi stage (owned = 0).
#include <cuda_runtime.h>

#include <algorithm>

#include "msv.cuh"
#include "vit.cuh"
#include "vit_pair.cuh"

namespace hmg {

// whole-warp MSV registers that cover a model of up to 32*QV nodes (2*32*QL >= 32*QV + 1)
// whole-warp MSV registers for a model of M nodes: 2 * 32 * QL >= M + 1
int long_msv_q(int M) { return (M + (kMsvQPlus1 ? 1 : 0) + 63) / 64; }   // 2 x 32 x QL >= M (msv.cuh)

template <int QL>
__global__ void __launch_bounds__(256) pipe_long_msv_kernel(const LongArgs A) {
  constexpr int WM = kRows * QL * 32;
  extern __shared__ uint4 smem4[];
  {
    const uint4* s0 = reinterpret_cast<const uint4*>(A.m.prof);
    for (int i = threadIdx.x; i < WM / 4; i += blockDim.x) smem4[i] = s0[i];
  }
  __syncthreads();
  const uint32_t* smm = reinterpret_cast<const uint32_t*>(smem4);
  const int lane = threadIdx.x & 31;
  for (;;) {
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(A.counter, 1ull);
    b = __shfl_sync(0xffffffffu, b, 0);
    if ((long long)b >= A.nitems) break;
    // item -> (sequence j, chunk c): chunk_start is the exclusive prefix of chunks per sequence
    int lo = 0, hi = (int)A.nlong;             // largest j with chunk_start[j] <= b
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if ((unsigned long long)A.chunk_start[mid] <= b) lo = mid;
      else hi = mid;
    }
    const int j = lo;
    const int c = (int)(b - A.chunk_start[j]);
    const int nch = A.chunk_start[j + 1] - A.chunk_start[j];
    const int L = A.m.len[j];
    const int r0 = c * A.chunk_rows;
    const int r1 = min(L, r0 + A.chunk_rows);
    int rm = 0;
    const bool ok = msv_chunk<QL>(A.m, smm, j, r0, r1, A.m.M, &rm);
    if (lane == 0) {
      A.chunk_max[b] = ok ? rm : -1;
      __threadfence();
    }
    unsigned prev = 0;
    if (lane == 0) prev = atomicAdd(A.chunk_done + j, 1u);
    prev = __shfl_sync(0xffffffffu, prev, 0);
    if ((int)prev != nch - 1) continue;          // not the last chunk of sequence j
    __threadfence();
    // last finisher: combine, or fall back to the sequential DP
    int Rmax = 0;
    bool all_ok = true;
    for (int k = A.chunk_start[j] + lane; k < A.chunk_start[j + 1]; k += 32) {
      const int v = *((volatile int*)A.chunk_max + k);
      if (v < 0) all_ok = false;
      Rmax = max(Rmax, v);
    }
    all_ok = __all_sync(0xffffffffu, all_ok);
    Rmax = __reduce_max_sync(0xffffffffu, Rmax);
    int raw;
    if (all_ok) {
      const int tjb = A.m.tjb[L];
      const int Bp = min(max(kBaseB - tjb - A.m.tbm, 0) + A.m.bias, 255);
      raw = Rmax > Bp ? max(Rmax - A.m.bias - 3, 0) : 254;
      if (lane == 0) A.m.raw[j] = (uint8_t)raw;
    } else {
      // the chunk that called for this re-run saw a crossing, so a branch-free pass first would be
      // wasted: short rows (QL <= 4) vote once per word (msv_batch<32, QL>), longer ones run the
      // checked pass only -- the per-word vote's register snapshot costs 28-30 registers in this
      // kernel (fewer resident chunk warps).  Measured (profiles/cmp_r02zt.jsonl, ms per step):
      // checked 5.80 / 2.99 / 7.27 / 15.61, per-word vote 5.88 / 2.82 / 7.00 / 15.81 on configs
      // 3 (QL = 7) / 2 (QL = 4) / 5 at M = 100 (QL = 2) / 5 at M = 500 (QL = 8)
      if constexpr (QL <= 4) raw = msv_batch<32, QL>(A.m, smm, (long long)j, A.nlong);
      else raw = msv_batch<32, QL, false, true>(A.m, smm, (long long)j, A.nlong);   // sequential DP
    }
    if (lane == 0) A.owned[j] = raw != 254;
  }
}


// Viterbi filter of the long sequences that passed MSV (pipeline only): one warp per sequence,
// longest first, on blocks that each ask for most of an SM's shared memory (so they hold their
// SMs alone).  Every block executes griddepcontrol.launch_dependents as soon as it is resident;
// the main MSV kernel is launched next in the same stream with programmatic stream
// serialisation, so it is dispatched only after these blocks are placed and then fills the
// other SMs while this kernel runs.  Its inputs (raw MSV scores of the long sequences) come
// from pipe_long_msv_kernel, which completed before it in stream order: nothing waits on a
// concurrently running kernel, so serialised execution (profilers, sanitizers) stays correct.
template <int QV>
__global__ void __launch_bounds__(128) pipe_long_vit_kernel(const LongArgs A) {
  asm volatile("griddepcontrol.launch_dependents;");
  constexpr int WV = kRows * QV * 32;
  extern __shared__ uint4 smem4[];
  {
    const uint4* s1 = reinterpret_cast<const uint4*>(A.v.rsc);
    for (int i = threadIdx.x; i < WV / 4; i += blockDim.x) smem4[i] = s1[i];
  }
  __syncthreads();
  const int32_t* smv = reinterpret_cast<const int32_t*>(smem4);
  const int lane = threadIdx.x & 31;
  VitLane<32, QV, true> V;
  V.load(A.v.tr, lane);
  for (;;) {
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(A.counter + 1, 1ull);
    b = __shfl_sync(0xffffffffu, b, 0);
    if ((long long)b >= A.nlong) break;
    const int j = (int)b;
    if (!A.owned[j]) continue;                   // 254: the exact re-score + main stage decide
    const int raw = A.m.raw[j];
    const int L = A.m.len[j];
    if (!(raw == 255 || raw >= (int)A.thr[L])) continue;       // MSV pass flag (reading R25)
    const uint32_t* wp = A.v.words + (size_t)A.v.woff16[j] * 4;
    V.start(A.v.move[L], true);
    ResStream rs;
    rs.init(wp, (L + 5) / 6);
    for (int iq = 0; iq < rs.nq; ++iq) {                        // Alg 2 row loop
      uint4 w4 = rs.next(iq);
#pragma unroll 1
      for (int k = 0; k < 4; ++k) {
        const uint32_t w = w4.x;
        w4.x = w4.y;
        w4.y = w4.z;
        w4.z = w4.w;
#pragma unroll
        for (int jj = 0; jj < 6; ++jj) {
          const int x = (w >> (5 * jj)) & 31;
          V.row(smv + x * (QV * 32), lane, 0xffffffffu);
        }
      }
    }
    const int vraw = V.finish();
    if (lane == 0) A.v.raw_sorted[j] = (int16_t)vraw;
  }
}

template <int Q>
__global__ void __launch_bounds__(128) pipe_long_vpair_kernel(const LongArgs A) {
  asm volatile("griddepcontrol.launch_dependents;");
  constexpr int WV = kRows * Q * 32;
  extern __shared__ uint4 smem4[];
  {
    const uint4* s1 = reinterpret_cast<const uint4*>(A.v.rsc);
    for (int i = threadIdx.x; i < WV / 4; i += blockDim.x) smem4[i] = s1[i];
  }
  __syncthreads();
  const uint32_t* smv = reinterpret_cast<const uint32_t*>(smem4);
  const uint32_t* tr = reinterpret_cast<const uint32_t*>(A.v.tr);
  const int lane = threadIdx.x & 31;
  // (measured slower here: the max-plus scan Lazy-F, 387 -> 559 cycles per lone row at
  //  M = 400, and a latency row form with the carries exchanged in the first Lazy-F round)
  VitPairLane<32, Q> V;
  V.load(tr, lane);
  for (;;) {
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(A.counter + 1, 1ull);
    b = __shfl_sync(0xffffffffu, b, 0);
    if ((long long)b >= A.nlong) break;
    const int j = (int)b;
    if (!A.owned[j]) continue;                   // 254: the exact re-score + main stage decide
    const int raw = A.m.raw[j];
    const int L = A.m.len[j];
    if (!(raw == 255 || raw >= (int)A.thr[L])) continue;       // MSV pass flag (reading R25)
    const uint32_t* wp = A.v.words + (size_t)A.v.woff16[j] * 4;
    V.start(tr, lane, A.v.move[L], A.v.tbm_min, A.v.safe, true, 0xffffffffu);
    ResStream rs;
    rs.init(wp, (L + 5) / 6);
    for (int iq = 0; iq < rs.nq; ++iq) {                        // Alg 2 row loop
      uint4 w4 = rs.next(iq);
#pragma unroll 1
      for (int k = 0; k < 4; ++k) {
        const uint32_t w = w4.x;
        w4.x = w4.y;
        w4.y = w4.z;
        w4.z = w4.w;
#pragma unroll
        for (int jj = 0; jj < 6; ++jj) {
          const int x = (w >> (5 * jj)) & 31;
          V.row(smv + x * (Q * 32), tr, lane, 0xffffffffu);
        }
      }
    }
    const int vraw = V.finish();
    if (lane == 0) {
      if (vraw >= -32768) A.v.raw_sorted[j] = (int16_t)vraw;
      else A.owned[j] = 0;                       // outside the window: the main stage scores it
    }
  }
}

namespace {
template <int Q>
const void* pick_vpair(int q) {
  if constexpr (Q > 16) {
    return nullptr;
  } else {
    if (q == Q) return reinterpret_cast<const void*>(&pipe_long_vpair_kernel<Q>);
    return pick_vpair<Q + 1>(q);
  }
}
template <int QV>
const void* pick_vit(int q) {
  if constexpr (QV > 16) {
    return nullptr;
  } else {
    if (q == QV) return reinterpret_cast<const void*>(&pipe_long_vit_kernel<QV>);
    return pick_vit<QV + 1>(q);
  }
}
template <int QL>
const void* pick_msv(int q) {
  if constexpr (QL > 17) {   // models up to 1024 nodes
    return nullptr;
  } else {
    if (q == QL) return reinterpret_cast<const void*>(&pipe_long_msv_kernel<QL>);
    return pick_msv<QL + 1>(q);
  }
}
}  // namespace

cudaError_t launch_pipe_long_msv(int QL, const LongArgs& a, cudaStream_t st, int* ok) {
  const void* fn = pick_msv<1>(QL);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = (size_t)kRows * QL * 32 * 4;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 256, smem);
  if (e != cudaSuccess) return e;
  const int64_t need = (a.nitems + 7) / 8;
  int64_t grid = std::min<int64_t>((int64_t)nsm * std::max(per, 1), std::max<int64_t>(need, 1));
  void* args[] = {const_cast<LongArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(256), args, smem, st);
}

}  // namespace hmg

namespace hmg {
cudaError_t launch_pipe_long_vit(int QV, bool pair, const LongArgs& a, int nblocks, cudaStream_t st, int* ok) {
  const void* fn = pair ? pick_vpair<1>(QV) : pick_vit<1>(QV);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t need = (size_t)kRows * QV * 32 * 4;
  int dev = 0, maxsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const size_t smem = std::max(need, (size_t)maxsm - 8192);   // hold the SM alone
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  void* args[] = {const_cast<LongArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)nblocks), dim3(128), args, smem, st);
}
}  // namespace hmg
