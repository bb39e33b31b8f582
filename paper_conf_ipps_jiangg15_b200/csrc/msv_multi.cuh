// msv_multi.cuh -- many-profile MSV (an hmmscan/Pfam-style batch, many profiles
// x one DB stream per launch; Pfam scale P:819-824).
//
// msv_multi_kernel<G, Q>: one launch scores every (profile, sequence) pair of a bucket of
// profiles that share the lane geometry (G lanes x Q s16x2 registers; smaller profiles are
// padded with -inf nodes, which never contribute).  The length-sorted DB is cut into chunks of
// C sequences; a block takes work items (chunk c, profile p) from an atomic queue in
// chunk-major order, stages profile p's striped table in shared memory and its 8 warps score
// the chunk's sequences with msv_batch<G, Q> (the single-profile lane code, unchanged) from a
// block-local counter.  Chunk-major order starts the longest sequences of every profile first
// and keeps a chunk's residues in L2 while all profiles read them (the DB crosses HBM once
// per chunk instead of once per profile).
#pragma once
#include "msv.cuh"

namespace hmg {

template <int G, int Q>
__device__ __forceinline__ void msv_multi_body(const MsvMultiArgs& m) {
  extern __shared__ uint4 smem4[];
  __shared__ long long item_sh;
  __shared__ unsigned sub_ctr;
  constexpr int W0 = MsvLayout<G, Q>::WORDS;
  constexpr int NG = 32 / G;
  const uint32_t* sm = reinterpret_cast<const uint32_t*>(smem4);
  const int lane = threadIdx.x & 31;
  const long long nitems = m.nchunks * (long long)m.nprof;
  for (;;) {
    __syncthreads();                                   // previous item finished with the table
    if (threadIdx.x == 0) {
      item_sh = (long long)atomicAdd(m.counter, 1ull);
      sub_ctr = 0;
    }
    __syncthreads();
    const long long item = item_sh;
    if (item >= nitems) break;
    const long long c = item / m.nprof;
    const int p = (int)(item % m.nprof);
    {
      const uint4* src = reinterpret_cast<const uint4*>(m.prof[p]);
      for (int i = threadIdx.x; i < W0 / 4; i += blockDim.x) smem4[i] = src[i];
    }
    __syncthreads();
    MsvArgs a = m.base;
    a.bias = m.bias[p];
    a.tbm = m.tbm[p];
    a.raw = m.raw + (size_t)p * (size_t)m.base.nseq;
    const long long lo = c * m.chunk;
    const long long hi = min(lo + (long long)m.chunk, (long long)m.base.nseq);
    for (;;) {
      unsigned b = 0;
      if (lane == 0) b = atomicAdd(&sub_ctr, (unsigned)NG);
      b = __shfl_sync(0xffffffffu, b, 0);
      if (lo + (long long)b >= hi) break;
      msv_batch<G, Q>(a, sm, lo + (long long)b, hi);
    }
  }
}

template <int G, int Q>
__global__ void __launch_bounds__(256) msv_multi_kernel(const MsvMultiArgs m) { msv_multi_body<G, Q>(m); }

template <int G, int Q, int MB>
__global__ void __launch_bounds__(256, MB) msv_multi_kernel_mb(const MsvMultiArgs m) { msv_multi_body<G, Q>(m); }

// the same per-geometry minimum-blocks policy as the single-profile kernel (msv_min_blocks)
template <int G, int Q>
const void* msv_multi_entry() {
  constexpr int MB = msv_min_blocks<G, Q>();
  if constexpr (MB > 0) return reinterpret_cast<const void*>(&msv_multi_kernel_mb<G, Q, MB>);
  else return reinterpret_cast<const void*>(&msv_multi_kernel<G, Q>);
}

}  // namespace hmg
