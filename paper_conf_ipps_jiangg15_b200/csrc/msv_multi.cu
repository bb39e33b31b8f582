// msv_multi.cu -- many-profile MSV: launcher of msv_multi_kernel<G, Q>, the exact
// re-score over (profile, sequence) pairs, and the batched pass-flag epilogue.
//
// The exact pair kernel is Alg 1 with u8 saturation, like msv_exact_kernel, one warp
// per pair; it serves the rare pairs the fast lanes flag (raw 254: every cell <= B', all-gap or
// extremely low-scoring sequences).
#include <cuda_runtime.h>

#include <algorithm>

#include "msv.cuh"

namespace hmg {

const void* msv_multi_ptr_g4(int q);
const void* msv_multi_ptr_g8(int q);
const void* msv_multi_ptr_g16(int q);
const void* msv_multi_ptr_g32(int q);

static const void* msv_multi_ptr(int G, int Q) {
  switch (G) {
    case 4: return msv_multi_ptr_g4(Q);
    case 8: return msv_multi_ptr_g8(Q);
    case 16: return msv_multi_ptr_g16(Q);
    case 32: return msv_multi_ptr_g32(Q);
  }
  return nullptr;
}

cudaError_t launch_msv_multi(int G, int Q, const MsvMultiArgs& a, cudaStream_t st, int* ok) {
  const void* fn = msv_multi_ptr(G, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = (size_t)msv_table_words(G, Q) * 4;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 256, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  long long grid = (long long)nsm * per;
  const long long items = a.nchunks * (long long)a.nprof;
  if (grid > items) grid = items;
  if (grid < 1) grid = 1;
  void* args[] = {const_cast<MsvMultiArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(256), args, smem, st);
}

__device__ __forceinline__ int u8s(int v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

__global__ void __launch_bounds__(256) msv_pairs_exact_kernel(const MsvPairArgs a) {
  const int lane = threadIdx.x & 31;
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  uint8_t* prev = a.scratch + (size_t)warp * 2 * (a.Mmax + 1);
  uint8_t* cur = prev + (a.Mmax + 1);
  const long long n = *a.nlist;
  for (long long idx = warp; idx < n; idx += nwarps) {
    const long long j = a.list[idx];
    const int p = (int)(j / a.nseq);
    const int s = (int)(j % a.nseq);
    const int M = a.M[p], bias = a.bias[p], tbm = a.tbm[p];
    const uint8_t* cost = a.cost[p];
    const int L = a.len[s];
    const int tjb = a.tjb[L];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    for (int k = lane; k <= M; k += 32) prev[k] = 0;            // Alg 1 l.9
    if (lane == 0) cur[0] = 0;
    __syncwarp();
    int xJ = 0, xB = u8s(kBaseB - tjb), raw = -1;
    uint8_t* pr = prev;
    uint8_t* cu = cur;
    for (int i = 0; i < L; ++i) {
      const int x = (__ldg(wp + i / 6) >> (5 * (i % 6))) & 31;
      const int xBp = u8s(xB - tbm);
      int xE = 0;
      const uint8_t* crow = cost + (size_t)x * M;
      for (int k = 1 + lane; k <= M; k += 32) {                 // Alg 1 l.14-16
        int v = max((int)pr[k - 1], xBp);
        v = u8s(v + bias);
        v = u8s(v - (int)__ldg(crow + k - 1));
        cu[k] = (uint8_t)v;
        xE = max(xE, v);
      }
      xE = __reduce_max_sync(0xffffffffu, xE);
      __syncwarp();
      if (xE >= 255 - bias) { raw = 255; break; }                // reading R13
      xJ = max(xJ, u8s(xE - 3));
      xB = u8s(max(xJ, kBaseB) - tjb);
      uint8_t* t = pr; pr = cu; cu = t;
    }
    if (lane == 0) a.raw[(size_t)p * a.nseq + s] = (uint8_t)(raw < 0 ? xJ : raw);
    __syncwarp();
  }
}

cudaError_t launch_msv_pairs_exact(const MsvPairArgs& a, int nwarps, cudaStream_t st) {
  g_launches += 1;
  msv_pairs_exact_kernel<<<(nwarps * 32 + 255) / 256, 256, 0, st>>>(a);
  return cudaGetLastError();
}

// Pairs the fast lanes flagged 254 (and every pair of a profile outside the fast kernel's
// precondition, pre-set to 254), appended by a grid-wide ballot/atomic (order does not matter:
// each entry is an independent pair, p * nseq + s with p the row in bucket order).
__global__ void append_254_kernel(const uint8_t* __restrict__ raw, int64_t n, int64_t* __restrict__ list,
                                  unsigned long long* __restrict__ ctr) {
  const int lane = threadIdx.x & 31;
  for (int64_t c0 = (int64_t)blockIdx.x * blockDim.x; c0 < n; c0 += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = c0 + threadIdx.x;
    const bool f = k < n && raw[k] == 254;
    const unsigned bal = __ballot_sync(0xffffffffu, f);
    if (!bal) continue;
    unsigned long long w0 = 0;
    if (lane == 0) w0 = atomicAdd(ctr, (unsigned long long)__popc(bal));
    w0 = __shfl_sync(0xffffffffu, w0, 0);
    if (f) list[w0 + __popc(bal & ((1u << lane) - 1u))] = k;
  }
}

cudaError_t select_redo_pairs(const uint8_t* raw_sorted, int64_t n, int64_t* list, int64_t* count,
                              cudaStream_t st) {
  // count lives in the first 8 bytes of `count` storage: reuse it as the append counter
  unsigned long long* ctr = reinterpret_cast<unsigned long long*>(count);
  cudaError_t e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long), st);
  if (e != cudaSuccess) return e;
  if (n > 0) {
    int64_t b = (n + 255) / 256;
    if (b > 148 * 16) b = 148 * 16;
    g_launches += 1;
    append_254_kernel<<<(unsigned)b, 256, 0, st>>>(raw_sorted, n, list, ctr);
  }
  return cudaGetLastError();
}

// raw [p][s] sorted order -> caller order, pass = overflow or raw >= thr_p[L] (reading R25)
__global__ void msv_flags_multi_kernel(const uint8_t* __restrict__ raw, int nprof, const int32_t* __restrict__ len,
                                       const int32_t* __restrict__ order, int64_t nseq,
                                       const uint16_t* const* __restrict__ thr, const int* __restrict__ rowmap,
                                       uint8_t* __restrict__ raw_out, uint8_t* __restrict__ pass_out,
                                       uint8_t* __restrict__ pass_sorted) {
  const int p = blockIdx.y;                    // row of raw (bucket order) -> caller profile rowmap[p]
  const uint8_t* r = raw + (size_t)p * nseq;
  const uint16_t* th = thr ? thr[p] : nullptr;
  const size_t ro = (size_t)rowmap[p] * nseq;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nseq; k += (int64_t)gridDim.x * blockDim.x) {
    const int v = r[k];
    const size_t c = ro + order[k];
    raw_out[c] = (uint8_t)v;
    const uint8_t pv = th ? (uint8_t)(v == 255 || v >= (int)th[len[k]]) : 0;
    if (pass_out) pass_out[c] = pv;
    if (pass_sorted) pass_sorted[(size_t)p * nseq + k] = pv;   // row p (bucket order), sorted order
  }
}

cudaError_t msv_flags_multi(const uint8_t* raw_sorted, int nprof, const int32_t* len, const int32_t* order,
                            int64_t nseq, const uint16_t* const* thr, const int* rowmap, uint8_t* raw_out,
                            uint8_t* pass_out, cudaStream_t st, uint8_t* pass_sorted) {
  if (nseq <= 0 || nprof <= 0) return cudaSuccess;
  int64_t bx = (nseq + 255) / 256;
  const int64_t cap = std::max<int64_t>(1, 4096 / nprof);
  if (bx > cap) bx = cap;
  g_launches += 1;
  msv_flags_multi_kernel<<<dim3((unsigned)bx, (unsigned)nprof), 256, 0, st>>>(raw_sorted, nprof, len, order, nseq,
                                                                             thr, rowmap, raw_out, pass_out,
                                                                             pass_sorted);
  return cudaGetLastError();
}

}  // namespace hmg
