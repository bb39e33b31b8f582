// pipeline.cu -- pass flags, on-device stable survivor compaction and caller-order scatter.
//
// Fig 1: every sequence goes through MSV, ~2.2% pass on to
// P7Viterbi.  The paper does not say how survivors reach the
// second stage; here the MSV pass flags are evaluated on the device against a
// per-length integer threshold table (built on the host from the Gumbel tail,
// P:41-45, reading R25) and the passing sequences are compacted with a stable
// three-kernel scan (count per tile, scan of tile counts, scatter), so the
// survivor list keeps the length-descending schedule order and no host
// round-trip sits between the two filters.
#include <cuda_runtime.h>

#include "hmg_internal.h"

namespace hmg {

constexpr int kTile = 4096;      // elements per compaction tile
constexpr int kThreads = 256;    // 16 elements per thread

size_t scan_tmp_bytes(int64_t n) {
  const int64_t nt = (n + kTile - 1) / kTile + 1;
  return (size_t)(2 * nt + 2) * sizeof(int64_t);
}

// Row y = blockIdx.y of a [rows][n] flag matrix (one row for the single-profile calls): flags at
// y * n, tile counts / offsets at y * tstride, outputs of caller row rowmap[y] (rowmap NULL: y).
__global__ void count_kernel(const uint8_t* __restrict__ flag, int64_t n, int64_t* __restrict__ tilecnt,
                             int64_t tstride) {
  flag += (size_t)blockIdx.y * n;
  tilecnt += (size_t)blockIdx.y * tstride;
  const int64_t t0 = (int64_t)blockIdx.x * kTile;
  int c = 0;
  for (int i = threadIdx.x; i < kTile; i += kThreads) {
    const int64_t k = t0 + i;
    if (k < n && flag[k]) ++c;
  }
  c = __reduce_add_sync(0xffffffffu, c);
  __shared__ int ws[kThreads / 32];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    int tot = 0;
    for (int w = 0; w < kThreads / 32; ++w) tot += ws[w];
    tilecnt[blockIdx.x] = tot;
  }
}

// exclusive scan of tile counts by one block; writes total to *count
__global__ void scan_kernel(const int64_t* __restrict__ tilecnt, int64_t ntiles, int64_t* __restrict__ tileoff,
                            int64_t* __restrict__ count, int64_t tstride, const int* __restrict__ rowmap) {
  tilecnt += (size_t)blockIdx.x * tstride;
  tileoff += (size_t)blockIdx.x * tstride;
  count += rowmap ? rowmap[blockIdx.x] : (int)blockIdx.x;
  __shared__ int64_t carry;
  __shared__ int64_t wsum[kThreads / 32];
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t b = 0; b < ntiles; b += kThreads) {
    const int64_t i = b + threadIdx.x;
    int64_t v = (i < ntiles) ? tilecnt[i] : 0;
    // inclusive warp scan
    int64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if ((threadIdx.x & 31) >= o) x += y;
    }
    if ((threadIdx.x & 31) == 31) wsum[threadIdx.x >> 5] = x;
    __syncthreads();
    int64_t wo = 0;
    for (int w = 0; w < (int)(threadIdx.x >> 5); ++w) wo += wsum[w];
    if (i < ntiles) tileoff[i] = carry + wo + x - v;
    __syncthreads();
    if (threadIdx.x == kThreads - 1) carry += wo + x;
    __syncthreads();
  }
  if (threadIdx.x == 0) *count = carry;
}

// stable scatter: ids_sorted[j] = k, ids_caller[j] = order[k] for the j-th flagged k
__global__ void scatter_kernel(const uint8_t* __restrict__ flag, int64_t n, const int64_t* __restrict__ tileoff,
                               const int32_t* __restrict__ order, int32_t* __restrict__ ids_sorted,
                               int32_t* __restrict__ ids_caller, int64_t tstride, const int* __restrict__ rowmap) {
  flag += (size_t)blockIdx.y * n;
  tileoff += (size_t)blockIdx.y * tstride;
  if (ids_sorted) ids_sorted += (size_t)blockIdx.y * n;
  if (ids_caller) ids_caller += (size_t)(rowmap ? rowmap[blockIdx.y] : (int)blockIdx.y) * n;
  const int64_t t0 = (int64_t)blockIdx.x * kTile;
  __shared__ int64_t base;
  __shared__ int wsum[kThreads / 32];
  if (threadIdx.x == 0) base = tileoff[blockIdx.x];
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int c0 = 0; c0 < kTile; c0 += kThreads) {
    const int64_t k = t0 + c0 + threadIdx.x;
    const bool f = k < n && flag[k];
    const unsigned bal = __ballot_sync(0xffffffffu, f);
    if (lane == 0) wsum[w] = __popc(bal);
    __syncthreads();
    int wo = 0, tot = 0;
    for (int i = 0; i < kThreads / 32; ++i) {
      if (i < w) wo += wsum[i];
      tot += wsum[i];
    }
    if (f) {
      const int64_t j = base + wo + __popc(bal & ((1u << lane) - 1u));
      if (ids_sorted) ids_sorted[j] = (int32_t)k;
      if (ids_caller) ids_caller[j] = order[k];
    }
    __syncthreads();
    if (threadIdx.x == 0) base += tot;
    __syncthreads();
  }
}

static cudaError_t compact(const uint8_t* flag, int64_t n, const int32_t* order, int32_t* ids_sorted,
                           int32_t* ids_caller, int64_t* count, void* tmp, cudaStream_t st) {
  const int64_t nt = (n + kTile - 1) / kTile;
  int64_t* tilecnt = reinterpret_cast<int64_t*>(tmp);
  int64_t* tileoff = tilecnt + nt + 1;
  if (nt == 0) return cudaMemsetAsync(count, 0, sizeof(int64_t), st);
  g_launches += 1;
  count_kernel<<<(unsigned)nt, kThreads, 0, st>>>(flag, n, tilecnt, 0);
  g_launches += 1;
  scan_kernel<<<1, kThreads, 0, st>>>(tilecnt, nt, tileoff, count, 0, nullptr);
  g_launches += 1;
  scatter_kernel<<<(unsigned)nt, kThreads, 0, st>>>(flag, n, tileoff, order, ids_sorted, ids_caller, 0, nullptr);
  return cudaGetLastError();
}

size_t compact_rows_tmp_bytes(int64_t n, int rows) {
  const int64_t nt = (n + kTile - 1) / kTile;
  return (size_t)rows * 2 * (size_t)(nt + 1) * sizeof(int64_t) + 16;
}

// Stable compaction of every row of a [rows][n] sorted-order flag matrix in three launches
// (many-profile pipeline): ids_sorted [rows][n] (row y), ids_caller / counts at caller row rowmap[y].
cudaError_t compact_rows(const uint8_t* flag, int rows, int64_t n, const int32_t* order, int32_t* ids_sorted,
                         int32_t* ids_caller, int64_t* counts, const int* rowmap, void* tmp, cudaStream_t st) {
  const int64_t nt = (n + kTile - 1) / kTile;
  if (rows <= 0) return cudaSuccess;
  const int64_t ts = nt + 1;
  int64_t* tilecnt = reinterpret_cast<int64_t*>(tmp);
  int64_t* tileoff = tilecnt + (size_t)rows * ts;
  if (nt == 0) return cudaSuccess;
  g_launches += 1;
  count_kernel<<<dim3((unsigned)nt, (unsigned)rows), kThreads, 0, st>>>(flag, n, tilecnt, ts);
  g_launches += 1;
  scan_kernel<<<(unsigned)rows, kThreads, 0, st>>>(tilecnt, nt, tileoff, counts, ts, rowmap);
  g_launches += 1;
  scatter_kernel<<<dim3((unsigned)nt, (unsigned)rows), kThreads, 0, st>>>(flag, n, tileoff, order, ids_sorted,
                                                                          ids_caller, ts, rowmap);
  return cudaGetLastError();
}

// stable compaction of a sorted-order flag array (Viterbi passes -> Forward list)
cudaError_t compact_flags(const uint8_t* flag_sorted, int64_t n, const int32_t* order, int32_t* ids_sorted,
                          int32_t* ids_caller, int64_t* count, void* tmp, cudaStream_t st) {
  return compact(flag_sorted, n, order, ids_sorted, ids_caller, count, tmp, st);
}

__global__ void redo_flag_kernel(const uint8_t* __restrict__ raw, int64_t n, uint8_t* __restrict__ flag) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x)
    flag[k] = raw[k] == 254;
}

cudaError_t select_redo(const uint8_t* raw_sorted, int64_t n, int32_t* list, int64_t* count, void* tmp,
                        cudaStream_t st) {
  uint8_t* flag = reinterpret_cast<uint8_t*>(reinterpret_cast<char*>(tmp) + scan_tmp_bytes(n));
  if (n > 0) {
    g_launches += 1;
    const int64_t b = (n + 1023) / 1024;
    redo_flag_kernel<<<(unsigned)(b < 4096 ? b : 4096), 1024, 0, st>>>(raw_sorted, n, flag);
  }
  return compact(flag, n, nullptr, list, nullptr, count, tmp, st);
}

// MSV epilogue: scatter raw to caller order, pass = overflow or raw >= thr[L] (reading R25)
__global__ void msv_flag_kernel(const uint8_t* __restrict__ raw, const int32_t* __restrict__ len,
                                const int32_t* __restrict__ order, int64_t n, const uint16_t* __restrict__ thr,
                                uint8_t* __restrict__ raw_out, uint8_t* __restrict__ pass_out,
                                uint8_t* __restrict__ flag) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const int r = raw[k];
    const int c = order[k];
    const uint8_t p = thr ? (uint8_t)(r == 255 || r >= (int)thr[len[k]]) : 0;
    raw_out[c] = (uint8_t)r;
    if (pass_out) pass_out[c] = p;
    flag[k] = p;
  }
}

cudaError_t msv_finish(const uint8_t* raw_sorted, const int32_t* len, const int32_t* order, int64_t n,
                       const uint16_t* thr, uint8_t* raw_out, uint8_t* pass_out, int32_t* surv_sorted,
                       int64_t* nsurv, int32_t* surv_caller, void* tmp, cudaStream_t st) {
  uint8_t* flag = reinterpret_cast<uint8_t*>(reinterpret_cast<char*>(tmp) + scan_tmp_bytes(n));
  if (n > 0) {
    const int64_t b = (n + 255) / 256;
    g_launches += 1;
    msv_flag_kernel<<<(unsigned)(b < 8192 ? b : 8192), 256, 0, st>>>(raw_sorted, len, order, n, thr, raw_out,
                                                                      pass_out, flag);
  }
  if (!surv_sorted && !surv_caller) return cudaGetLastError();
  return compact(flag, n, order, surv_sorted, surv_caller, nsurv, tmp, st);
}

__global__ void vit_flag_kernel(const int16_t* __restrict__ raw, const int32_t* __restrict__ list,
                                const int64_t* __restrict__ nlist, int64_t nmax, const int32_t* __restrict__ len,
                                const int32_t* __restrict__ order, const int32_t* __restrict__ thr,
                                int16_t* __restrict__ raw_out, uint8_t* __restrict__ pass_out,
                                uint8_t* __restrict__ flags_out, uint8_t* __restrict__ pass_sorted) {
  const int64_t n = list ? *nlist : nmax;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    const int s = list ? list[j] : (int)j;
    const int r = raw[s];
    const int c = order[s];
    raw_out[c] = (int16_t)r;
    const bool p = thr ? (r == 32767 || r >= thr[len[s]]) : false;
    if (pass_out) pass_out[c] = p;
    if (flags_out) flags_out[c] = (uint8_t)(flags_out[c] | 4u | (p ? 2u : 0u));
    if (pass_sorted) pass_sorted[s] = p;
  }
}

cudaError_t vit_finish(const int16_t* raw_sorted, const int32_t* list, const int64_t* nlist, int64_t nmax,
                       const int32_t* len, const int32_t* order, const int32_t* thr, int16_t* raw_out,
                       uint8_t* pass_out, uint8_t* flags_out, cudaStream_t st, uint8_t* pass_sorted) {
  if (nmax <= 0) return cudaSuccess;
  const int64_t b = (nmax + 255) / 256;
  g_launches += 1;
  vit_flag_kernel<<<(unsigned)(b < 8192 ? b : 8192), 256, 0, st>>>(raw_sorted, list, nlist, nmax, len, order, thr,
                                                                    raw_out, pass_out, flags_out, pass_sorted);
  return cudaGetLastError();
}

__global__ void to_sorted_kernel(const int32_t* __restrict__ caller, int64_t n, const int32_t* __restrict__ inv,
                                 int32_t* __restrict__ out) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    out[j] = inv[caller[j]];
}

cudaError_t to_sorted_ids(const int32_t* caller_ids, int64_t n, const int32_t* inv_order, int32_t* sorted_ids,
                          cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  const int64_t b = (n + 255) / 256;
  g_launches += 1;
  to_sorted_kernel<<<(unsigned)(b < 8192 ? b : 8192), 256, 0, st>>>(caller_ids, n, inv_order, sorted_ids);
  return cudaGetLastError();
}

__global__ void set_count_kernel(int64_t* d, int64_t v) { *d = v; }

cudaError_t set_count(int64_t* d, int64_t v, cudaStream_t st) {
  g_launches += 1;
  set_count_kernel<<<1, 1, 0, st>>>(d, v);
  return cudaGetLastError();
}

}  // namespace hmg
