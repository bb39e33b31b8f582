// vit_wide.cu -- instantiations and launcher of the one-warp long-model Viterbi kernel
// (vit_wide.cuh): Q = 8 .. 32 s16x2 registers per lane (models up to 64 Q nodes), transitions in
// shared memory (tm = false) or tensor memory (tm = true).
#include <cuda_runtime.h>

#include <algorithm>

#include "vit_wide.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pickw(int q, bool tm, size_t* smem, int* cols = nullptr) {
  if constexpr (Q > 32) {
    return nullptr;
  } else {
    if (q == Q) {
      *smem = tm ? VitWideSmem<Q, true>::bytes : VitWideSmem<Q, false>::bytes;
      if (cols) *cols = tm ? wide_tmem_cols<Q>() : 0;
      return tm ? reinterpret_cast<const void*>(&vit_wide_kernel<Q, true>)
                : reinterpret_cast<const void*>(&vit_wide_kernel<Q, false>);
    }
    return pickw<Q + 4>(q, tm, smem, cols);
  }
}
}  // namespace

bool vit_wide_available(int Q) {
  size_t b = 0;
  return Q % 4 == 0 && pickw<8>(Q, false, &b) != nullptr;
}
size_t vit_wide_smem(int Q, bool tm) {
  size_t b = 0;
  return pickw<8>(Q, tm, &b) ? b : 0;
}

cudaError_t launch_vit_wide(int Q, bool tm, const VitArgs& a, cudaStream_t st, int* ok) {
  size_t smem = 0;
  int cols = 0;
  const void* fn = Q % 4 == 0 ? pickw<8>(Q, tm, &smem, &cols) : nullptr;
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int nt = tm ? wide_threads<true>() : wide_threads<false>();
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, nt, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  if (cols > 0 && per * cols > 512) {
    // a CTA beyond the SM's 512 TMEM columns would wait in tcgen05.alloc for a whole resident
    // CTA (persistent) to finish: cap the residency with shared memory the kernel does not use
    per = 512 / cols;
    int maxsm = 0;
    cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    smem = std::max(smem, (size_t)(maxsm / (per + 1) + 1024));
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    if (smem > (size_t)optin) return cudaErrorInvalidConfiguration;
    if ((e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))) return e;
  }
  void* args[] = {const_cast<VitArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)(nsm * per)), dim3((unsigned)nt), args, smem, st);
}

}  // namespace hmg
