// msv.cu -- MSV launchers and the exact (general) MSV kernel.
//
// msv_exact_kernel is Alg 1 written with the byte arithmetic of
// the paper (u8 saturating max/add/sub, xE by warp max): one warp per
// sequence, lanes striding the model (the paper's "for p <- Idx; p < M;
// p += 32", Alg 1 l.14), DP row double-buffered in global scratch.  It runs
// only for profiles outside the fast kernel's precondition (bias >= 66 + tbm,
// which HMMER's background makes impossible for canonical profiles) and for
// the rare sequences the fast kernel flags (every cell <= B').
#include <cuda_runtime.h>

#include "msv.cuh"

namespace hmg {

const void* msv_fast_ptr_g4(int q);
const void* msv_fast_ptr_g8(int q);
const void* msv_fast_ptr_g16(int q);
const void* msv_fast_ptr_g32(int q);

int msv_q_max(int G) { return G == 32 ? 40 : 32; }

int msv_table_words(int G, int Q) { return MsvLayoutRT(G, Q).words; }

template <int G, int Q>
constexpr bool msv_layout_agrees() {
  constexpr MsvLayoutRT r(G, Q);
  using Lt = MsvLayout<G, Q>;
  return r.words == Lt::WORDS && r.stride == Lt::STRIDE && r.b2 == Lt::B2 && r.b1 == Lt::B1 &&
         (r.byte != 0) == Lt::BYTE && (!Lt::BYTE || Lt::NCB * G == 2 * G * Lt::NC2);   // byte chunk fits the slot
}
static_assert(msv_layout_agrees<4, 9>() && msv_layout_agrees<4, 10>() && msv_layout_agrees<8, 13>() &&
              msv_layout_agrees<8, 26>() && msv_layout_agrees<8, 7>() && msv_layout_agrees<16, 13>() &&
              msv_layout_agrees<16, 15>() && msv_layout_agrees<16, 18>() && msv_layout_agrees<32, 7>() &&
              msv_layout_agrees<32, 25>(), "MsvLayoutRT != MsvLayout");

static const void* msv_fast_ptr(int G, int Q) {
  switch (G) {
    case 4: return msv_fast_ptr_g4(Q);
    case 8: return msv_fast_ptr_g8(Q);
    case 16: return msv_fast_ptr_g16(Q);
    case 32: return msv_fast_ptr_g32(Q);
  }
  return nullptr;
}

cudaError_t launch_msv_fast(int G, int Q, const MsvArgs& a, cudaStream_t st, int* ok, bool pdl) {
  const void* fn = msv_fast_ptr(G, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const int QL = (G == 32) ? 0 : (G * Q + 31) / 32;
  const size_t smem = ((size_t)msv_table_words(G, Q) + (size_t)kRows * QL * 32) * 4;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 256, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  int64_t need = (a.nseq + (32 / G) * 8 - 1) / ((32 / G) * 8);   // blocks with any work
  int64_t grid = (int64_t)nsm * per;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  void* args[] = {const_cast<MsvArgs*>(&a)};
  g_launches += 1;
  if (!pdl) return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(256), args, smem, st);
  // programmatic dependent launch: may start once every block of the preceding kernel in the
  // stream (the pipeline long lane) is resident and has signalled griddepcontrol.launch_dependents
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, fn, args);
}

__device__ __forceinline__ int u8sat(int v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

__global__ void __launch_bounds__(256) msv_exact_kernel(const MsvArgs a) {
  const int lane = threadIdx.x & 31;
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  const int M = a.M, bias = a.bias, tbm = a.tbm;
  uint8_t* prev = a.scratch + (size_t)warp * 2 * (M + 1);
  uint8_t* cur = prev + (M + 1);
  const long long n = a.list ? *a.nlist : a.nseq;
  for (long long idx = warp; idx < n; idx += nwarps) {
    const int s = a.list ? a.list[idx] : (int)idx;
    const int L = a.len[s];
    const int tjb = a.tjb[L];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    for (int k = lane; k <= M; k += 32) prev[k] = 0;          // Alg 1 l.9
    if (lane == 0) cur[0] = 0;
    __syncwarp();
    int xJ = 0;
    int xB = u8sat(kBaseB - tjb);
    int raw = -1;
    uint8_t* p = prev;
    uint8_t* c = cur;
    for (int i = 0; i < L; ++i) {                             // Alg 1 l.10
      const int x = (__ldg(wp + i / 6) >> (5 * (i % 6))) & 31;  // l.11 decode
      const int xBp = u8sat(xB - tbm);
      int xE = 0;                                             // l.12
      const uint8_t* crow = a.cost + (size_t)x * M;
      for (int k = 1 + lane; k <= M; k += 32) {               // l.14
        int v = max((int)p[k - 1], xBp);                      // l.15
        v = u8sat(v + bias);
        v = u8sat(v - (int)__ldg(crow + k - 1));
        c[k] = (uint8_t)v;
        xE = max(xE, v);                                      // l.16
      }
      xE = __reduce_max_sync(0xffffffffu, xE);                // l.20 warp max
      __syncwarp();
      if (xE >= 255 - bias) { raw = 255; break; }
      xJ = max(xJ, u8sat(xE - 3));
      xB = u8sat(max(xJ, kBaseB) - tjb);
      uint8_t* t = p; p = c; c = t;
    }
    if (lane == 0) a.raw[s] = (uint8_t)(raw < 0 ? xJ : raw);  // l.23
    __syncwarp();
  }
}

cudaError_t launch_msv_exact(const MsvArgs& a, int nwarps, cudaStream_t st) {
  const int threads = 256;
  const int blocks = (nwarps * 32 + threads - 1) / threads;
  g_launches += 1;
  msv_exact_kernel<<<blocks, threads, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace hmg
