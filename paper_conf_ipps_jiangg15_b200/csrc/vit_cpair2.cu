// vit_cpair2.cu -- instantiations and launcher of the two-warp pair Viterbi kernel without a
// per-row block barrier (vit_cpair2.cuh): Q s16x2 registers per thread, SG sequences per block.
#include <cuda_runtime.h>

#include "vit_cpair2.cuh"

namespace hmg {
namespace {
template <int SG, int TSM, int Q, int QMAX>
const void* pick2(int q, size_t* smem) {
  if constexpr (Q > QMAX) {
    return nullptr;
  } else {
    if (q == Q) {
      *smem = VitCP2Smem<Q, SG, TSM>::bytes;
      return reinterpret_cast<const void*>(&vit_cpair2_kernel<Q, SG, TSM>);
    }
    return pick2<SG, TSM, Q + 1, QMAX>(q, smem);
  }
}
// variant = 10 * TSM + SG (TSM 2: tMM, tIM, tMI, tII streamed from shared memory)
const void* cpair2_ptr(int var, int Q, size_t* smem) {
  switch (var) {
    case 2: return pick2<2, 0, 2, 16>(Q, smem);
    case 12: return pick2<2, 1, 8, 16>(Q, smem);
    case 22: return pick2<2, 2, 2, 16>(Q, smem);
    case 23: return pick2<3, 2, 8, 16>(Q, smem);
  }
  return nullptr;
}
}  // namespace

size_t vit_cpair2_smem(int var, int Q) {
  size_t b = 0;
  return cpair2_ptr(var, Q, &b) ? b : 0;
}
bool vit_cpair2_available(int var, int Q) {
  size_t b = 0;
  return cpair2_ptr(var, Q, &b) != nullptr;
}

cudaError_t launch_vit_cpair2(int var, int Q, const VitArgs& a, cudaStream_t st, int* ok) {
  size_t smem = 0;
  const void* fn = cpair2_ptr(var, Q, &smem);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const int SG = var % 10;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 64 * SG, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  void* args[] = {const_cast<VitArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)(nsm * per)), dim3(64 * SG), args, smem, st);
}

}  // namespace hmg
