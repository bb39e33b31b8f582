// vit_pair.cu -- launcher of the s16x2 pair Viterbi kernel (vit_pair.cuh).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>

#include "vit_pair.cuh"

namespace hmg {

const void* vit_pair_ptr_g8(int q);
const void* vit_pair_ptr_g16(int q);
const void* vit_pair_ptr_g32(int q);
const void* vit_pair_ptr_g32s(int q);

int vit_pair_q_max() { return 16; }

static const void* vit_pair_ptr(int G, int Q, bool scan) {
  if (scan) return G == 32 ? vit_pair_ptr_g32s(Q) : nullptr;
  switch (G) {
    case 8: return vit_pair_ptr_g8(Q);
    case 16: return vit_pair_ptr_g16(Q);
    case 32: return vit_pair_ptr_g32(Q);
  }
  return nullptr;
}

cudaError_t launch_vit_pair(int G, int Q, bool scan, const VitArgs& a, cudaStream_t st, int* ok) {
  const void* fn = vit_pair_ptr(G, Q, scan);
  *ok = fn != nullptr;
  if (!fn) return cudaSuccess;
  const size_t smem = (((size_t)kRows * Q * G + 3) / 4) * 16;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, 128, smem);
  if (e != cudaSuccess) return e;
  if (per < 1) per = 1;
  // (fewer blocks per SM -- faster rows for the longest survivors, less throughput -- measured
  //  slower at 1 / 2 / 3 blocks: profiles/vit_bps_r01.jsonl)
  const int64_t grid = (int64_t)nsm * per;
  void* args[] = {const_cast<VitArgs*>(&a)};
  g_launches += 1;
  return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(128), args, smem, st);
}

}  // namespace hmg
