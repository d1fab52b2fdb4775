// Micro-benchmark: red.shared.add.u32 throughput (clk per warp-instruction per
// SM) for the narrow Q1 record pattern: 7 reductions per row to fields
// FSTRIDE bytes apart, optionally with shared loads in between.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/atoms_bench scripts/micro/atoms_bench.cu
#include <cstdint>
#include <cstdio>
template <int FSTRIDE, int LDS>
__global__ void k(int iters, unsigned long long* out) {
  extern __shared__ uint32_t sm[];
  for (int i = threadIdx.x; i < 7 * 7 * 512 + 4096; i += blockDim.x) sm[i] = 0;
  __syncthreads();
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(sm + threadIdx.x);
  const uint32_t l = (uint32_t)__cvta_generic_to_shared(sm + 7 * 7 * 512 + (threadIdx.x & 1023));
  uint32_t acc = 0;
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    uint32_t v = i;
#pragma unroll
    for (int j = 0; j < LDS; ++j) {
      uint32_t x;
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(x) : "r"(l + 4 * j));
      v += x;
    }
#pragma unroll
    for (int f = 0; f < 7; ++f) asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a + f * FSTRIDE), "r"(v) : "memory");
    acc += v;
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) atomicAdd(out, (unsigned long long)(t1 - t0) + (acc == 12345 ? 1 : 0));
}
template <int FSTRIDE, int LDS>
void run(const char* name, unsigned long long* d) {
  const int iters = 4096, threads = 512;
  cudaFuncSetAttribute(k<FSTRIDE, LDS>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaMemset(d, 0, 8);
  k<FSTRIDE, LDS><<<148, threads, (7 * 7 * 512 + 4096) * 4>>>(iters, d);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h;
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-40s %.3f clk per warp-ATOMS per SM (%s)\n", name, (double)h / 148 / ((double)iters * 7 * (threads / 32)),
         cudaGetErrorString(e));
}
int main() {
  unsigned long long* d;
  cudaMalloc(&d, 8);
  run<0, 0>("same word x7", d);
  run<2048, 0>("fields 2048 B apart (same bank)", d);
  run<2052, 0>("fields 2052 B apart (bank +1)", d);
  run<128, 0>("fields 128 B apart", d);
  run<2048, 1>("2048 B + 1 LDS per row", d);
  run<2048, 2>("2048 B + 2 LDS per row", d);
  return 0;
}
