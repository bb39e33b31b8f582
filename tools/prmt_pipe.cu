// Does PRMT share the ALU pipe with the DPX s16x2 ops?  Independent chains of PRMT, of
// VIADDMNMX.S16x2, and both interleaved (separate chains): if the mixed rate is the sum of the
// two, they issue on different pipes.  (Design probe for a byte-table MSV variant.)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define NC 8
#define IT 4096
template <int OP>
__global__ void k(uint32_t* out, uint32_t seed, uint32_t b, uint32_t c) {
  uint32_t r[NC], s[NC];
#pragma unroll
  for (int j = 0; j < NC; ++j) { r[j] = seed ^ (threadIdx.x * 7919u + j); s[j] = r[j] * 3u; }
  for (int it = 0; it < IT; ++it) {
#pragma unroll
    for (int j = 0; j < NC; ++j) {
      if (OP == 0 || OP == 2) r[j] = __viaddmax_s16x2(r[j], b, c);
      if (OP == 1 || OP == 2) s[j] = __byte_perm(s[j], b, 0x9180u + (j & 1));
    }
    b += 0x00010001u;
  }
  uint32_t acc = 0;
#pragma unroll
  for (int j = 0; j < NC; ++j) acc ^= r[j] ^ s[j];
  if (acc == 0x12345678u) out[0] = acc;
}
int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  uint32_t* d; cudaMalloc(&d, 64);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int blocks = p.multiProcessorCount * 8, threads = 256;
  const char* nm[] = {"VIADDMNMX.S16x2", "PRMT", "VIADDMNMX+PRMT (independent)"};
  for (int op = 0; op < 3; ++op)
    for (int rep = 0; rep < 3; ++rep) {
      cudaEventRecord(e0);
      if (op == 0) k<0><<<blocks, threads>>>(d, rep, 3, 5);
      if (op == 1) k<1><<<blocks, threads>>>(d, rep, 3, 5);
      if (op == 2) k<2><<<blocks, threads>>>(d, rep, 3, 5);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      const double ops = (double)blocks * threads * IT * NC * (op == 2 ? 2 : 1);
      if (rep == 2) printf("{\"op\": \"%s\", \"ms\": %.4f, \"T_lane_ops_per_s\": %.3f}\n", nm[op], ms, ops / ms / 1e9);
    }
  printf("{\"status\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
