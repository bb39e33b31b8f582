// vit_cpair.cu -- instantiations and launcher of the block-per-sequence pair Viterbi kernel
// (vit_cpair.cuh): W warps per sequence, Q s16x2 registers per thread and cell type.
#include <cuda_runtime.h>

#include "vit_cpair.cuh"

namespace hmg {
namespace {
// SG sequence groups of W warps share one block (and its shared-memory table)
template <int W, int SG, int Q, int QMAX>
const void* pick(int q) {
  if constexpr (Q > QMAX) {
    return nullptr;
  } else {
    if (q == Q) return reinterpret_cast<const void*>(&vit_cpair_kernel<W, Q, SG>);
    return pick<W, SG, Q + 1, QMAX>(q);
  }
}
const void* cpair_ptr(int W, int SG, int Q) {
  switch (W * 10 + SG) {
    case 22: return pick<2, 2, 8, 16>(Q);
    case 24: return pick<2, 4, 8, 16>(Q);
    case 41: return pick<4, 1, 2, 16>(Q);
    case 42: return pick<4, 2, 2, 16>(Q);
    case 43: return pick<4, 3, 2, 16>(Q);
    case 81: return pick<8, 1, 2, 8>(Q);
    case 82: return pick<8, 2, 2, 8>(Q);
    case 161: return pick<16, 1, 2, 4>(Q);
  }
  return nullptr;
}
}  // namespace

size_t vit_cpair_smem(int W, int SG, int Q) {
  const size_t tab = (size_t)21 * Q * 32 * W * 4;
  switch (W * 10 + SG) {
    case 22: return tab + sizeof(int) * VitCPairSmem<2, 1, 2>::NSCR;
    case 24: return tab + sizeof(int) * VitCPairSmem<2, 1, 4>::NSCR;
    case 41: return tab + sizeof(int) * VitCPairSmem<4, 1, 1>::NSCR;
    case 42: return tab + sizeof(int) * VitCPairSmem<4, 1, 2>::NSCR;
    case 43: return tab + sizeof(int) * VitCPairSmem<4, 1, 3>::NSCR;
    case 81: return tab + sizeof(int) * VitCPairSmem<8, 1, 1>::NSCR;
    case 82: return tab + sizeof(int) * VitCPairSmem<8, 1, 2>::NSCR;
    case 161: return tab + sizeof(int) * VitCPairSmem<16, 1, 1>::NSCR;
  }
  return 0;
}

bool vit_cpair_available(int W, int SG, int Q) { return cpair_ptr(W, SG, Q) != nullptr; }

cudaError_t launch_vit_cpair(int W, int SG, int Q, const VitArgs& a, cudaStream_t st, int* ok) {
  const void* fn = cpair_ptr(W, SG, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = vit_cpair_smem(W, SG, Q);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 32 * W * SG, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  void* args[] = {const_cast<VitArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)(nsm * per)), dim3(32 * W * SG), args, smem, st);
}

}  // namespace hmg
