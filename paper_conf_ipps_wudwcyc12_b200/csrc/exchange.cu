// exchange.cu — the device side of the multi-GPU SELECT exchange (SURVEY
// §8(a) a9, §8(e)).  Each rank selects from its own contiguous row range; after
// an all_gather of the per-rank counts, rank r's output belongs at the sum of
// the counts of ranks < r.  That is the paper's gather stage — matches must
// "determine their correct position in the final array" (Fig 3,
// L479-485) — one level up: ranks instead of CTA tiles.  The scan stays on the
// device and in stream order, so the next step never waits for the host.

#include "ra_internal.cuh"

namespace ra {
namespace {

// One warp: chunks of 32 counts, inclusive warp scan (shuffles), carry across
// chunks.  n_ranks is small (<= RA_MAX_RANKS): the cost is the launch.
__global__ void __launch_bounds__(32) offsets_kernel(const int64_t* __restrict__ counts, int n,
                                                     int64_t* __restrict__ offsets, int64_t* __restrict__ total) {
  dev::grid_dep_wait();
  const int lane = threadIdx.x;
  int64_t carry = 0;
  for (int base = 0; base < n; base += 32) {
    const int r = base + lane;
    const int64_t c = r < n ? counts[r] : 0;
    int64_t inc = c;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int64_t y = __shfl_up_sync(0xffffffffu, inc, d);
      if (lane >= d) inc += y;
    }
    if (r < n && offsets) offsets[r] = carry + inc - c;
    carry += __shfl_sync(0xffffffffu, inc, 31);
  }
  if (lane == 0 && total) *total = carry;
}

}  // namespace
}  // namespace ra

using namespace ra;

RA_API int ra_select_offsets(const int64_t* d_counts, int n_ranks, int64_t* d_offsets, int64_t* d_total,
                             ra_stream_t stream) {
  clear_error();
  if (n_ranks < 1 || n_ranks > RA_MAX_RANKS) return fail(RA_E_INVAL, "n_ranks=%d outside [1, %d]", n_ranks, RA_MAX_RANKS);
  if (!d_counts || (!d_offsets && !d_total)) return fail(RA_E_INVAL, "null argument");
  if (((uintptr_t)d_counts | (uintptr_t)d_offsets | (uintptr_t)d_total) & 7u)
    return fail(RA_E_INVAL, "pointers must be 8-byte aligned");
  cudaError_t e = launch_pdl(offsets_kernel, dim3(1), dim3(32), 0, (cudaStream_t)stream, d_counts, n_ranks,
                             d_offsets, d_total);
  count_launch();
  if (e != cudaSuccess) return cuda_fail(e, "offsets_kernel launch");
  return RA_OK;
}
