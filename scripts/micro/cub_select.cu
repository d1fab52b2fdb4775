// Yardstick: cub::DeviceSelect::If on 2^28 int32 (library routine; not product code).
#include <cub/cub.cuh>
#include <cstdio>
#include <cstdint>
#include <cstdlib>

struct LessThan {
  int32_t t;
  __host__ __device__ bool operator()(const int32_t& x) const { return x < t; }
};

__global__ void fill(int32_t* x, int64_t n, uint64_t seed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t z = seed + i * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    x[i] = (int32_t)(z >> 32);
  }
}

int main(int argc, char** argv) {
  const int lg = argc > 1 ? atoi(argv[1]) : 28;
  int64_t n = 1ll << lg;
  int32_t *x, *out; int* cnt;
  cudaMalloc(&x, n * 4); cudaMalloc(&out, n * 4); cudaMalloc(&cnt, 8);
  fill<<<1184, 256>>>(x, n, 7);
  for (double s : {0.01, 0.1, 0.25, 0.5, 0.75, 0.9}) {
    LessThan op{(int32_t)(-2147483648.0 + s * 4294967296.0)};
    size_t tb = 0; void* tmp = nullptr;
    cub::DeviceSelect::If(tmp, tb, x, out, cnt, (int)n, op);
    cudaMalloc(&tmp, tb);
    for (int i = 0; i < 3; ++i) cub::DeviceSelect::If(tmp, tb, x, out, cnt, (int)n, op);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    for (int i = 0; i < 20; ++i) cub::DeviceSelect::If(tmp, tb, x, out, cnt, (int)n, op);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); ms /= 20;
    int c; cudaMemcpy(&c, cnt, 4, cudaMemcpyDeviceToHost);
    printf("cub select 2^%d s=%.2f: %.4f ms  count %d  alg GB/s %.1f  (%s)\n", lg, s, ms, c, (4.0 * n + 4.0 * c) / ms / 1e6,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(tmp);
  }
  return 0;
}
