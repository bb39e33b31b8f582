// Instantiations and launcher of vit_cta_kernel<W, Q> (block-per-sequence Viterbi filter).
#include <cuda_runtime.h>

#include "vit_cta.cuh"

namespace hmg {
namespace {
template <int W, int Q>
const void* pick_q(int q) {
  if constexpr (Q > 8) {
    return nullptr;
  } else {
    if (q == Q) return reinterpret_cast<const void*>(&vit_cta_kernel<W, Q>);
    return pick_q<W, Q + 2>(q);
  }
}
const void* pick(int W, int Q) {
  switch (W) {
    case 4: return pick_q<4, 2>(Q);
    case 8: return pick_q<8, 2>(Q);
    case 16: return pick_q<16, 2>(Q);
  }
  return nullptr;
}
}  // namespace

size_t vit_cta_smem(int W, int Q) {
  // VitCtaSmem<W, Q>::table_bytes + NSCR ints
  return (size_t)21 * (Q / 2) * 32 * W * 4 + (size_t)(8 * W + 2 * W + 5 * W + 1) * 4;
}

cudaError_t launch_vit_cta(int W, int Q, const VitArgs& a, cudaStream_t st, int* ok) {
  const void* fn = pick(W, Q);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = vit_cta_smem(W, Q);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 32 * W, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  void* args[] = {const_cast<VitArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)(nsm * per)), dim3(32 * W), args, smem, st);
}

}  // namespace hmg
