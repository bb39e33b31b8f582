// tmem_bw.cu -- can tensor memory stand in for registers in a non-GEMM kernel?  Read throughput of
// tcgen05.ld (32x32b shapes: each lane reads consecutive 32-bit columns of its own TMEM row) per
// SM, alone and beside shared-memory LDS.128 traffic (the vit_wide kernel is LDS-bound on the
// transition vectors it streams from shared memory).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_bw tools/tmem_bw.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ void ld16(uint32_t a, uint32_t (&v)[16]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                 "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
               : "r"(a));
}
__device__ __forceinline__ void tm_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// MODE 0: TMEM only, 1: LDS only, 2: both (one LDS.128 per 16 TMEM words, the vit_wide mix:
// emission from shared memory, transitions from TMEM), 3: both, four LDS.128 per 16 TMEM words
template <int MODE, int COLS>
__global__ void __launch_bounds__(128) bw_kernel(int iters, uint32_t* out) {
  __shared__ uint32_t taddr_s;
  __shared__ __align__(16) uint32_t sm[4096];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = i * 2654435761u;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                 ::"r"((uint32_t)__cvta_generic_to_shared(&taddr_s)), "n"(COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t base = taddr_s + ((uint32_t)(warp * 32) << 16);   // lane quarter of this warp
  uint32_t acc = 0;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      if (MODE != 1) {
        uint32_t v[16];
        ld16(base + (uint32_t)((c * 16) % (COLS - 16)), v);
        tm_wait();
#pragma unroll
        for (int j = 0; j < 16; ++j) acc ^= v[j];
      }
      if (MODE != 0) {
        constexpr int NL = MODE == 3 ? 4 : 1;
#pragma unroll
        for (int l = 0; l < NL; ++l) {
          uint4 s;
          asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(s.x), "=r"(s.y), "=r"(s.z), "=r"(s.w)
                       : "r"(sbase + (uint32_t)((((c * 4 + l) * 32 + lane) * 16 + it * 64) & 16383)));
          acc ^= s.x ^ s.y ^ s.z ^ s.w;
        }
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr_s), "n"(COLS));
  if (acc == 0x12345678u) out[0] = acc;
}

template <int MODE, int COLS>
int run(int blocks_per_sm, const char* name) {
  int dev = 0, nsm = 0, clk = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  uint32_t* out;
  CK(cudaMalloc(&out, 4));
  const int iters = 20000;
  const int grid = nsm * blocks_per_sm;
  bw_kernel<MODE, COLS><<<grid, 128>>>(10, out);
  CK(cudaDeviceSynchronize());
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  bw_kernel<MODE, COLS><<<grid, 128>>>(iters, out);
  cudaEventRecord(b);
  CK(cudaEventSynchronize(b));
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  const double warps = (double)grid * 4;
  const double tm_bytes = MODE != 1 ? warps * iters * 8 * 32 * 16 * 4 : 0;
  const double ld_bytes = MODE != 0 ? warps * iters * 8 * 32 * 16 * (MODE == 3 ? 4 : 1) : 0;
  const double sm_clk = (double)nsm * ms * 1e-3 * 1e3 * (double)clk;   // SM-cycles at the nominal clock
  printf("{\"mode\": \"%s\", \"blocks_per_sm\": %d, \"ms\": %.3f, \"tmem_B_per_clk_sm\": %.1f, \"lds_B_per_clk_sm\": %.1f, \"tmem_TBps\": %.2f, \"lds_TBps\": %.2f}\n",
         name, blocks_per_sm, ms, tm_bytes / sm_clk, ld_bytes / sm_clk, tm_bytes / ms / 1e9, ld_bytes / ms / 1e9);
  cudaFree(out);
  return 0;
}

int main() {
  run<0, 128>(1, "tmem");
  run<0, 128>(2, "tmem");
  run<0, 128>(4, "tmem");
  run<1, 128>(2, "lds");
  run<1, 128>(4, "lds");
  run<2, 128>(2, "tmem+lds(1:4)");
  run<2, 128>(4, "tmem+lds(1:4)");
  run<3, 128>(2, "tmem+lds(1:1)");
  run<3, 128>(4, "tmem+lds(1:1)");
  return 0;
}
