// Dependent-chain latency (cycles from issue to a dependent issue) of the operations a lone
// long-lane warp serialises on per DP row: one warp, one chain, clock64 around
// ITERS dependent ops.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/oplat.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define ITERS 4096

template <int OP>
__global__ void lat(uint32_t* out, long long* cyc, uint32_t seed, uint32_t b, uint32_t c) {
  uint32_t r = seed ^ threadIdx.x;
  const long long t0 = clock64();
#pragma unroll 16
  for (int it = 0; it < ITERS; ++it) {
    if (OP == 0) r = __viaddmax_s16x2(r, b, c);                     // VIADDMNMX.S16x2
    if (OP == 1) r = __viaddmax_s16x2_relu(r, b, b);                // VIADDMNMX.S16x2.RELU
    if (OP == 2) r = __vimax3_s16x2(r, b, c);                       // VIMNMX3.S16x2
    if (OP == 3) r = __vmaxs2(r, b);                                // VIMNMX.S16x2
    if (OP == 4) r = r + b;                                         // IADD
    if (OP == 5) r = __byte_perm(r, b, 0x3210u ^ (it & 1));         // PRMT
    if (OP == 6) r = __shfl_sync(0xffffffffu, r, (threadIdx.x + 1) & 31) + b;   // SHFL.IDX (+ IADD)
    if (OP == 7) r = (uint32_t)__any_sync(0xffffffffu, (r & b) != 0u) + r;      // VOTE.ANY (+ ISETP, IADD)
    if (OP == 8) r = __ballot_sync(0xffffffffu, (r & b) != 0u) ^ r;             // VOTE.ALL ballot
    if (OP == 9) r = __reduce_or_sync(0xffffffffu, r & b) + r;                  // REDUX.OR (+ IADD)
    if (OP == 10) r = __viaddmax_s32(r, b, c);                      // VIADDMNMX (s32)
  }
  const long long t1 = clock64();
  if (r == 0x12345678u) out[0] = r;
  if (threadIdx.x == 0) cyc[OP] = t1 - t0;
}

template <int OP>
void run(uint32_t* d_out, long long* d_cyc) {
  lat<OP><<<1, 32>>>(d_out, d_cyc, 12345u, 0x00030005u, 0x7fff7fffu);
}

int main() {
  uint32_t* d_out;
  long long* d_cyc;
  cudaMalloc(&d_out, 4);
  cudaMalloc(&d_cyc, 16 * sizeof(long long));
  const char* names[] = {"VIADDMNMX.S16x2", "VIADDMNMX.S16x2.RELU", "VIMNMX3.S16x2", "VIMNMX.S16x2", "IADD",
                         "PRMT", "SHFL.IDX+IADD", "VOTE.ANY+ISETP+IADD", "ballot+ISETP+LOP", "REDUX.OR+IADD",
                         "VIADDMNMX.S32"};
  for (int rep = 0; rep < 2; ++rep) {
    run<0>(d_out, d_cyc); run<1>(d_out, d_cyc); run<2>(d_out, d_cyc); run<3>(d_out, d_cyc);
    run<4>(d_out, d_cyc); run<5>(d_out, d_cyc); run<6>(d_out, d_cyc); run<7>(d_out, d_cyc);
    run<8>(d_out, d_cyc); run<9>(d_out, d_cyc); run<10>(d_out, d_cyc);
    cudaDeviceSynchronize();
  }
  long long cyc[16];
  cudaMemcpy(cyc, d_cyc, sizeof(cyc), cudaMemcpyDeviceToHost);
  for (int i = 0; i < 11; ++i)
    printf("{\"op\": \"%s\", \"cycles_per_dependent_op\": %.2f}\n", names[i], (double)cyc[i] / ITERS);
  printf("{\"status\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
