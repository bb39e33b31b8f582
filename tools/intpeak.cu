// Integer-SIMD issue-rate microbenchmark for sm_100a (B200).
// Measures lane-ops/clk/SM for the DPX / s16x2 instructions the MSV and
// Viterbi-filter kernels are built from, so the roofline in DESIGN.md is a
// measured number rather than a guess.  Each kernel runs NCHAIN independent
// dependency chains per thread (ILP) so the pipe, not latency, is the limit.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define NCHAIN 8
#define ITERS 4096

template <int OP>
__global__ void bench(uint32_t* out, uint32_t seed, uint32_t b, uint32_t c) {
  uint32_t r[NCHAIN];
#pragma unroll
  for (int j = 0; j < NCHAIN; ++j) r[j] = seed ^ (threadIdx.x * 7919u + j);
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int j = 0; j < NCHAIN; ++j) {
      if (OP == 0) r[j] = __viaddmax_s16x2(r[j], b, c);            // VIADDMNMX.S16x2
      if (OP == 1) r[j] = __vimax3_s16x2(r[j], b, c);              // VIMNMX3.S16x2
      if (OP == 2) r[j] = __vmaxs2(r[j], b);                        // VIMNMX.S16x2
      if (OP == 3) r[j] = __vadd2(r[j], b);                         // VIADD.16x2
      if (OP == 4) r[j] = __viaddmax_s32(r[j], b, c);              // VIADDMNMX (s32)
      if (OP == 5) r[j] = r[j] + b;                                 // IADD3 / IMAD.IADD
      if (OP == 6) { r[j] = __viaddmax_s16x2(r[j], b, c); r[j] = __vimax3_s16x2(r[j], b ^ j, c); } // mix
      if (OP == 7) { r[j] = __viaddmax_s16x2(r[j], b, c); r[j] = r[j] + (b ^ j); } // DPX + int add mix
    }
    b += 0x00010001u;
  }
  uint32_t acc = 0;
#pragma unroll
  for (int j = 0; j < NCHAIN; ++j) acc ^= r[j];
  if (acc == 0x12345678u) out[0] = acc;
}

// shared-memory LDS.128 bandwidth: each thread reads 16 B per access, conflict-free.
__global__ void lds128(uint32_t* out, int iters) {
  extern __shared__ uint4 sm[];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = make_uint4(i, i * 3, i * 5, i * 7);
  __syncthreads();
  uint32_t acc = 0;
  int idx = threadIdx.x & 1023;
  for (int it = 0; it < iters; ++it) {
    uint4 v = sm[(idx + it * 32) & 4095];
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678u) out[0] = acc;
}

int main() {
  int dev = 0; cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
  int clk_khz = 0; cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"clock_khz_attr\": %d}\n", p.name, p.multiProcessorCount, clk_khz);
  uint32_t* d; cudaMalloc(&d, 64);
  const char* names[] = {"VIADDMNMX.S16x2", "VIMNMX3.S16x2", "VIMNMX.S16x2", "VIADD.16x2",
                         "VIADDMNMX.S32", "IADD", "VIADDMNMX+VIMNMX3", "VIADDMNMX+IADD"};
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int blocks = p.multiProcessorCount * 8, threads = 256;
  for (int op = 0; op < 8; ++op) {
    for (int rep = 0; rep < 3; ++rep) {
      cudaEventRecord(e0);
      switch (op) {
        case 0: bench<0><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 1: bench<1><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 2: bench<2><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 3: bench<3><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 4: bench<4><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 5: bench<5><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 6: bench<6><<<blocks, threads>>>(d, rep, 3, 5); break;
        case 7: bench<7><<<blocks, threads>>>(d, rep, 3, 5); break;
      }
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double instr = (double)blocks * threads * ITERS * NCHAIN * ((op >= 6) ? 2 : 1);
      if (rep == 2)
        printf("{\"op\": \"%s\", \"ms\": %.4f, \"Tlaneops_per_s\": %.3f}\n", names[op], ms, instr / ms / 1e9);
    }
  }
  cudaFuncSetAttribute(lds128, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  for (int rep = 0; rep < 3; ++rep) {
    int iters = 1 << 16;
    cudaEventRecord(e0);
    lds128<<<blocks, threads, 65536>>>(d, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double bytes = (double)blocks * threads * iters * 16;
    if (rep == 2) printf("{\"op\": \"LDS.128\", \"ms\": %.4f, \"TB_per_s\": %.3f}\n", ms, bytes / ms / 1e9);
  }
  cudaError_t err = cudaGetLastError();
  printf("{\"status\": \"%s\"}\n", cudaGetErrorString(err));
  return 0;
}
