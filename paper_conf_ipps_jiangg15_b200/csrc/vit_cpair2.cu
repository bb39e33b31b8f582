// vit_cpair2.cu -- instantiations and launcher of the two-warp pair Viterbi kernel without a
// per-row block barrier (vit_cpair2.cuh): Q s16x2 registers per thread, SG sequences per block.
#include <cuda_runtime.h>

#include "vit_cpair2.cuh"

namespace hmg {
namespace {
template <int SG, int Q, int QMAX>
const void* pick2(int q) {
  if constexpr (Q > QMAX) {
    return nullptr;
  } else {
    if (q == Q) return reinterpret_cast<const void*>(&vit_cpair2_kernel<Q, SG>);
    return pick2<SG, Q + 1, QMAX>(q);
  }
}
const void* cpair2_ptr(int SG, int Q) {
  switch (SG) {
    case 1: return pick2<1, 8, 16>(Q);
    case 2: return pick2<2, 2, 16>(Q);
    case 3: return pick2<3, 8, 16>(Q);
  }
  return nullptr;
}
size_t cpair2_smem(int SG, int Q) {
  const size_t tab = (size_t)21 * Q * 64 * 4;
  const size_t grp = sizeof(uint32_t) * ((Q * 64 + 16 + 2 + 2 + 3) / 4 * 4);
  return tab + sizeof(uint32_t) * 4 + (size_t)SG * grp;
}
}  // namespace

size_t vit_cpair2_smem(int SG, int Q) { return cpair2_ptr(SG, Q) ? cpair2_smem(SG, Q) : 0; }
bool vit_cpair2_available(int SG, int Q) { return cpair2_ptr(SG, Q) != nullptr; }

cudaError_t launch_vit_cpair2(int SG, int Q, const VitArgs& a, cudaStream_t st, int* ok) {
  const void* fn = cpair2_ptr(SG, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = cpair2_smem(SG, Q);
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
