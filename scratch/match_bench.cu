#include <cstdio>
#include <cstdint>
__global__ void k_match(uint32_t* out, int iters, uint32_t seed) {
  uint32_t x = seed ^ (threadIdx.x * 2654435761u) ^ blockIdx.x;
  uint32_t acc = 0;
  for (int i = 0; i < iters; ++i) {
    x = x * 1664525u + 1013904223u;
    uint32_t d = (x >> 13) & 255u;
    uint32_t peers = __match_any_sync(0xffffffffu, d);
    acc += __popc(peers & ((1u << (threadIdx.x & 31)) - 1u));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_ballot(uint32_t* out, int iters, uint32_t seed) {
  uint32_t x = seed ^ (threadIdx.x * 2654435761u) ^ blockIdx.x;
  uint32_t acc = 0;
  for (int i = 0; i < iters; ++i) {
    x = x * 1664525u + 1013904223u;
    uint32_t d = (x >> 13) & 255u;
    uint32_t peers = 0xffffffffu;
#pragma unroll
    for (int b = 0; b < 8; ++b) { uint32_t bal = __ballot_sync(0xffffffffu, (d >> b) & 1); peers &= ((d >> b) & 1) ? bal : ~bal; }
    acc += __popc(peers & ((1u << (threadIdx.x & 31)) - 1u));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_base(uint32_t* out, int iters, uint32_t seed) {
  uint32_t x = seed ^ (threadIdx.x * 2654435761u) ^ blockIdx.x;
  uint32_t acc = 0;
  for (int i = 0; i < iters; ++i) {
    x = x * 1664525u + 1013904223u;
    uint32_t d = (x >> 13) & 255u;
    acc += __popc(d & ((1u << (threadIdx.x & 31)) - 1u));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
int main() {
  uint32_t* out; cudaMalloc(&out, 148*16*256*4);
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  int iters = 4096; int grid = 148*8;
  for (int k = 0; k < 3; ++k) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(a);
      if (k==0) k_match<<<grid,256>>>(out, iters, rep);
      if (k==1) k_ballot<<<grid,256>>>(out, iters, rep);
      if (k==2) k_base<<<grid,256>>>(out, iters, rep);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      double warp_ops = (double)grid*8*iters;
      if (rep) printf("%s: %.3f ms, %.2f warp-ops/clk/SM (at 1.9GHz)\n", k==0?"match":k==1?"ballot8":"base", ms, warp_ops/(ms*1e-3)/148/1.9e9);
    }
  }
  return 0;
}
