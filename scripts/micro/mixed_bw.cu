// Microbenchmark (not product code): HBM bandwidth of a read stream that also
// writes a fraction of what it reads, like a SELECT at selectivity w (4 B in,
// 4w B out per row).  Persistent CTAs, 2 per SM, each streaming 32 KB chunks
// through a 2-slot cp.async.bulk ring; per chunk the CTA writes the first
// w * 32 KB of the chunk to a contiguous output range with coalesced 128-bit
// stores.  Reports (read + write bytes) / time.
//   usage: mixed_bw   (sweeps w = 0, 1/8, 1/4, 1/2, 1)
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

constexpr int CHUNK = 32768;
constexpr int DEPTH = 2;
constexpr int NT = 256;

__global__ void __launch_bounds__(NT, 2) mixed(const char* __restrict__ src, size_t nbytes, int4* __restrict__ dst,
                                               int wbytes) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint64_t bar[DEPTH];
  const size_t nchunks = nbytes / CHUNK;
  if (threadIdx.x == 0) {
    for (int s = 0; s < DEPTH; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  auto issue = [&](size_t c, int s) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])), "r"(CHUNK)
                 : "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(sm + s * CHUNK)),
        "l"(src + c * CHUNK), "r"(CHUNK), "r"(smem_u32(&bar[s]))
        : "memory");
  };
  if (threadIdx.x == 0)
    for (int s = 0; s < DEPTH && blockIdx.x + (size_t)s * gridDim.x < nchunks; ++s)
      issue(blockIdx.x + (size_t)s * gridDim.x, s);
  size_t i = 0;
  for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++i) {
    const int s = i % DEPTH;
    const uint32_t par = (i / DEPTH) & 1;
    asm volatile("{.reg .pred p; W%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W%=;}" ::"r"(
                     smem_u32(&bar[s])),
                 "r"(par)
                 : "memory");
    const int4* in = reinterpret_cast<const int4*>(sm + s * CHUNK);
    int4* out = dst + c * (size_t)(wbytes / 16);
    for (int e = threadIdx.x; e < wbytes / 16; e += NT) out[e] = in[e];
    __syncthreads();
    if (threadIdx.x == 0) {
      const size_t cn = c + (size_t)DEPTH * gridDim.x;
      if (cn < nchunks) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(cn, s);
      }
    }
  }
}

int main() {
  const size_t n = 1ull << 30;  // bytes read per launch
  char* src;
  int4* dst;
  cudaMalloc(&src, n);
  cudaMalloc(&dst, n);
  cudaMemset(src, 1, n);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaFuncSetAttribute(mixed, cudaFuncAttributeMaxDynamicSharedMemorySize, DEPTH * CHUNK);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int fr[] = {0, 4096, 8192, 16384, 32768};
  for (int wb : fr) {
    for (int rep = 0; rep < 3; ++rep) mixed<<<2 * sms, NT, DEPTH * CHUNK>>>(src, n, dst, wb);
    cudaEventRecord(a);
    const int reps = 20;
    for (int rep = 0; rep < reps; ++rep) mixed<<<2 * sms, NT, DEPTH * CHUNK>>>(src, n, dst, wb);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    ms /= reps;
    const double w = (double)wb / CHUNK;
    printf("write/read %.3f : %.4f ms  read %.0f GB/s  read+write %.0f GB/s  %s\n", w, ms, n / ms / 1e6,
           n * (1 + w) / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
