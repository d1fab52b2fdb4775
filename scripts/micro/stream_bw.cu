// Microbenchmark: how fast can one persistent CTA/SM stream HBM into shared
// memory with cp.async.bulk (varying chunk size / ring depth / CTAs per SM),
// versus plain LDG.128?  Not product code.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int CHUNK, int DEPTH>
__global__ void bulk_stream(const char* __restrict__ src, size_t nbytes, unsigned long long* sink) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint64_t bar[DEPTH];
  const size_t nchunks = nbytes / CHUNK;
  if (threadIdx.x == 0) {
    for (int s = 0; s < DEPTH; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  auto issue = [&](size_t c, int s) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])), "r"(CHUNK) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(sm + s * CHUNK)), "l"(src + c * CHUNK), "r"(CHUNK), "r"(smem_u32(&bar[s])) : "memory");
  };
  size_t i = 0;
  unsigned long long acc = 0;
  if (threadIdx.x == 0)
    for (int s = 0; s < DEPTH && blockIdx.x + (size_t)s * gridDim.x < nchunks; ++s) issue(blockIdx.x + (size_t)s * gridDim.x, s);
  for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++i) {
    const int s = i % DEPTH;
    const uint32_t par = (i / DEPTH) & 1;
    asm volatile("{.reg .pred p; W%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W%=;}" ::"r"(smem_u32(&bar[s])), "r"(par) : "memory");
    acc += ((const int*)(sm + s * CHUNK))[threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0) {
      size_t cn = c + (size_t)DEPTH * gridDim.x;
      if (cn < nchunks) { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); issue(cn, s); }
    }
  }
  if (acc == 0x12345) *sink = acc;
}

template <int UNROLL>
__global__ void ldg_stream(const int4* __restrict__ src, size_t n16, unsigned long long* sink) {
  unsigned long long acc = 0;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + (UNROLL - 1) * stride < n16; i += UNROLL * stride) {
    int4 v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(src + i + u * stride));
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) acc += v[u].x ^ v[u].w;
  }
  if (acc == 0x12345) *sink = acc;
}

template <typename F>
float timeit(F f) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) f();
  cudaEventRecord(a);
  for (int i = 0; i < 10; ++i) f();
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / 10;
}

template <int CHUNK, int DEPTH>
void run_bulk(const char* d, size_t nbytes, unsigned long long* sink, int ctas_per_sm, int threads) {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  size_t smem = (size_t)CHUNK * DEPTH;
  cudaFuncSetAttribute(bulk_stream<CHUNK, DEPTH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  float ms = timeit([&] { bulk_stream<CHUNK, DEPTH><<<sms * ctas_per_sm, threads, smem>>>(d, nbytes, sink); });
  cudaError_t e = cudaGetLastError();
  printf("bulk chunk=%6d depth=%d ctas/sm=%d thr=%d : %8.1f GB/s %s\n", CHUNK, DEPTH, ctas_per_sm, threads, nbytes / ms / 1e6, e ? cudaGetErrorString(e) : "");
}

int main() {
  size_t nbytes = 1ull << 30;
  char* d; cudaMalloc(&d, nbytes); cudaMemset(d, 1, nbytes);
  unsigned long long* sink; cudaMalloc(&sink, 8);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  // in-flight sweep: bytes in flight per SM = chunk * depth * ctas
  run_bulk<16384, 1>(d, nbytes, sink, 1, 256);
  run_bulk<16384, 2>(d, nbytes, sink, 1, 256);
  run_bulk<16384, 3>(d, nbytes, sink, 1, 256);
  run_bulk<16384, 4>(d, nbytes, sink, 1, 256);
  run_bulk<16384, 6>(d, nbytes, sink, 1, 256);
  run_bulk<16384, 8>(d, nbytes, sink, 1, 256);
  run_bulk<16384, 2>(d, nbytes, sink, 2, 256);
  run_bulk<16384, 3>(d, nbytes, sink, 2, 256);
  run_bulk<16384, 4>(d, nbytes, sink, 2, 256);
  run_bulk<32768, 2>(d, nbytes, sink, 1, 256);
  run_bulk<32768, 3>(d, nbytes, sink, 1, 256);
  run_bulk<32768, 2>(d, nbytes, sink, 2, 288);
  run_bulk<32768, 3>(d, nbytes, sink, 2, 288);
  for (int per = 2; per <= 8; per *= 2) {
    float ms = timeit([&] { ldg_stream<4><<<sms * per, 256>>>((const int4*)d, nbytes / 16, sink); });
    printf("ldg unroll4 ctas/sm=%d : %8.1f GB/s\n", per, nbytes / ms / 1e6);
    ms = timeit([&] { ldg_stream<8><<<sms * per, 256>>>((const int4*)d, nbytes / 16, sink); });
    printf("ldg unroll8 ctas/sm=%d : %8.1f GB/s\n", per, nbytes / ms / 1e6);
  }
  {
    char* o; cudaMalloc(&o, nbytes);
    float ms = timeit([&] { cudaMemcpyAsync(o, d, nbytes, cudaMemcpyDeviceToDevice); });
    printf("cudaMemcpy D2D 1 GiB: %8.1f GB/s (read+write)\n", 2.0 * nbytes / ms / 1e6);
  }
  return 0;
}
