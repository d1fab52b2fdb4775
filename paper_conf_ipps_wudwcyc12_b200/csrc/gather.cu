// gather.cu — the gather stage of a tuple SELECT (ra_select_rows, SURVEY
// §8(f) f3): out_j[i] = col_j[ids[i]] for every payload field j and every
// selected row i < min(*d_count, cap).
//
// The fused select kernel compacts the selected rows' ids in one pass
// (select_fused.cu, ROWS mode).  Gathering payload fields inside that
// kernel's write stage puts a dependent global load on the compute warps'
// critical path every tile (measured: 3 int32 fields at 2^28 rows, k=2,
// s=.5: 1.06 ms); this kernel instead runs the gather with the whole GPU's
// memory-level parallelism: each thread keeps GATHER_U ids x m fields of
// independent loads in flight, ids and outputs are coalesced across lanes,
// and the count is read on the device (no host round trip).  This is the
// paper's stage 4 "gather" (Fig 3) as its own kernel, as in the
// paper, but after a single-pass compaction instead of a global sync.
#include "ra_internal.cuh"

namespace ra {
namespace {

constexpr int GATHER_T = 256;
constexpr int GATHER_U = 4;

#ifndef RA_GATHER_LD
#define RA_GATHER_LD 2  // 0: __ldg; 1: ld.global.nc.L1::no_allocate; 2: + .L2::64B prefetch-size hint (measured: 897 -> 489 MB of DRAM reads at s=.01)
#endif
// One payload element at a random row: each touches its own sector, so L1
// allocation buys nothing and the L2 fetch granularity decides the DRAM bytes.
__device__ __forceinline__ uint32_t ld_gather32(const uint32_t* p) {
#if RA_GATHER_LD == 1
  uint32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#elif RA_GATHER_LD == 2
  uint32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}
__device__ __forceinline__ unsigned long long ld_gather64(const unsigned long long* p) {
#if RA_GATHER_LD == 1
  unsigned long long v;
  asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
#elif RA_GATHER_LD == 2
  unsigned long long v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}

__global__ void __launch_bounds__(GATHER_T) gather_kernel(const uint32_t* __restrict__ ids,
                                                          const int64_t* __restrict__ d_count, int64_t cap,
                                                          const GatherSpec g) {
  dev::grid_dep_wait();
  int64_t cnt = *d_count;
  if (cnt * g.sparse_den > g.n) return;  // dense: compact_kernel places the fields
  if (cnt > cap) cnt = cap;
  const int64_t step = (int64_t)gridDim.x * GATHER_T * GATHER_U;
  for (int64_t base = (int64_t)blockIdx.x * GATHER_T * GATHER_U; base < cnt; base += step) {
    uint32_t id[GATHER_U];
#pragma unroll
    for (int u = 0; u < GATHER_U; ++u) {
      const int64_t i = base + u * GATHER_T + threadIdx.x;
      id[u] = i < cnt ? __ldg(ids + i) : 0u;
    }
    uint64_t v[RA_MAX_PAYLOAD][GATHER_U];
#pragma unroll
    for (int j = 0; j < RA_MAX_PAYLOAD; ++j) {
      if (j < g.m) {  // uniform
#pragma unroll
        for (int u = 0; u < GATHER_U; ++u) {
          const bool ok = base + u * GATHER_T + threadIdx.x < cnt;
          v[j][u] = !ok ? 0ull
                    : g.elem_bytes[j] == 4 ? (uint64_t)ld_gather32((const uint32_t*)g.col[j] + id[u])
                                           : (uint64_t)ld_gather64((const unsigned long long*)g.col[j] + id[u]);
        }
      }
    }
#pragma unroll
    for (int j = 0; j < RA_MAX_PAYLOAD; ++j) {
      if (j < g.m) {
#pragma unroll
        for (int u = 0; u < GATHER_U; ++u) {
          const int64_t i = base + u * GATHER_T + threadIdx.x;
          if (i < cnt) {
            if (g.elem_bytes[j] == 4)
              ((uint32_t*)g.out[j])[i] = (uint32_t)v[j][u];
            else
              ((uint64_t*)g.out[j])[i] = v[j][u];
          }
        }
      }
    }
  }
}

}  // namespace

int launch_gather(const uint32_t* ids, const int64_t* d_count, int64_t cap, const GatherSpec& g, cudaStream_t s) {
  if (g.m == 0 || cap == 0) return RA_OK;
  int64_t grid = (cap + GATHER_T * GATHER_U - 1) / (GATHER_T * GATHER_U);
  const int64_t lim = (int64_t)num_sms() * 8;
  if (grid > lim) grid = lim;
  cudaError_t e = launch_pdl(gather_kernel, dim3((unsigned)grid), dim3(GATHER_T), 0, s, ids, d_count, cap, g);
  count_launch();
  if (e != cudaSuccess) return cuda_fail(e, "gather_kernel launch");
  return RA_OK;
}

}  // namespace ra
