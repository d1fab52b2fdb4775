// ra_internal.cuh — shared internals of libra.so (product side only; the
// oracle shares none of this).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <mutex>
#include <utility>

#include "ra.h"

#define RA_API extern "C" __attribute__((visibility("default")))

namespace ra {

// ------------------------------------------------------------ errors
int fail(int code, const char* fmt, ...);  // sets the thread-local message, returns code
int cuda_fail(cudaError_t e, const char* what);
void clear_error();

extern std::atomic<uint64_t> g_launches;
inline void count_launch(uint64_t k = 1) { g_launches.fetch_add(k, std::memory_order_relaxed); }

int num_sms();  // of the current device (cached per device)

// The current CUDA device, clamped to the 64 per-device cache slots.
int current_device();

// Per-device lazy initialisation (kernel attributes, occupancy, SM count):
// the first caller computes the value under one process-wide mutex, later
// callers read it lock-free (acquire/release), so concurrent first calls from
// several host threads are safe (ra.h: calls are reentrant).  `compute`
// returns a value > 0, or a negative RA_E_* code (not cached).
std::mutex& init_mutex();
template <typename F>
int device_once(std::atomic<int>* slots, int dev, F&& compute) {
  int v = slots[dev].load(std::memory_order_acquire);
  if (v > 0) return v;
  std::lock_guard<std::mutex> g(init_mutex());
  v = slots[dev].load(std::memory_order_relaxed);
  if (v > 0) return v;
  v = compute();
  if (v > 0) slots[dev].store(v, std::memory_order_release);
  return v;
}

// Launch with programmatic stream serialization (see dev::grid_dep_wait).
template <typename... Params, typename... Args>
cudaError_t launch_pdl(void (*kern)(Params...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                       Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// ------------------------------------------------- predicate canonical form
// A conjunction of k (op, value) predicates on a signed int32 equals
//   lo <= x <= hi  and  x != ne[0..n_ne)
// (an empty interval when lo > hi).  Folding the chain once on the host is the
// Table III observation: the fused "d<T1 && d<T2" compiles
// to the instructions of a single compare.
struct CanonPred {
  int32_t lo, hi;
  int32_t n_ne;
  int32_t ne[RA_MAX_PREDS];
};
int canonicalize(const ra_pred* preds, int k, CanonPred* out);

// ------------------------------------------------------------ SELECT
constexpr int SEL_THREADS = 256;  // compute threads per CTA (plus one look-back warp)
#ifndef RA_SEL_VEC  // (overridable for scripts/micro sweeps only)
#define RA_SEL_VEC 8
#define RA_SEL_AHEAD 1
#define RA_SEL_OUTRING 10240
#endif
constexpr int SEL_VEC = RA_SEL_VEC;      // int4 vectors per compute thread per tile
constexpr int SEL_AHEAD = RA_SEL_AHEAD;  // tiles whose bulk copy is in flight ahead of the count
constexpr int SEL_INSLOTS = SEL_AHEAD + 1;           // input ring slots (tiles)
constexpr int SEL_OUTRING = RA_SEL_OUTRING;          // compacted-row ring (int32), 40 KB
constexpr int SEL_TILE = SEL_THREADS * SEL_VEC * 4;  // 8192 rows / tile
int sel_ctas_per_sm();  // occupancy of the select kernel on the current device

// Workspace layout (see select_fused.cu):
//   [0, 256)                       header (launch epoch)
//   [256, 256 + 8 * ntiles)        status words (epoch-tagged)
//   [W - inter, W)                 unfused only: two int32[n] + 2 int64 counts
constexpr size_t SEL_HDR_BYTES = 256;
int64_t sel_max_tiles(int64_t n);  // tiles for n rows with any 16-B misalignment
size_t sel_status_bytes(int64_t n);
size_t sel_inter_bytes(int64_t n);

// One single-output select pass (select_fused_kernel: the unfused chain's
// passes and the tuple SELECT's key pass).  n_max = host bound on rows; d_n
// (nullable) = device-resident actual row count (<= n_max) produced by a
// previous pass.  rows != nullptr: row-id mode (the selected rows' ids go to
// rows[0..out_cap), d_out unused).
// Row-id mode extras for the payload compaction (compact.cu), per select tile t
// (SEL_TILE rows counted from the key's 16-B aligned base): the compute lanes'
// flag words fmask[t*SEL_THREADS + tid] and a 48-B record meta[t*12 ..]: the
// compute warps' exclusive bases within the tile (u32 [0..8)) and the tile's
// output offset (int64 at u32 index 8).
struct SelMasks {
  uint32_t* fmask;
  uint32_t* meta;
};
size_t sel_masks_bytes(int64_t n);

int launch_select_pass(const int32_t* d_in, int64_t n_max, const int64_t* d_n, const CanonPred& cp,
                       int32_t* d_out, int64_t out_cap, int64_t* d_count, void* d_ws,
                       cudaStream_t s, uint32_t* rows = nullptr, const SelMasks* masks = nullptr);

// Several SELECTs on one input in one pass (select_multi.cu), 1 <= M <= 4:
// cp[o] = output o's folded chain; validated arguments.
// d_n (nullable): device-resident row count (<= n) of the input, from a previous pass.
int launch_select_multi(const int32_t* d_in, int64_t n, const CanonPred* cp, int M, int32_t* const* d_outs,
                        const int64_t* out_caps, int64_t* const* d_counts, void* d_ws, cudaStream_t s,
                        const int64_t* d_n = nullptr);
size_t mo_workspace_bytes(int64_t n);

// Payload fields of a tuple SELECT.  The selectivity decides, on the device,
// which of the two kernels launched back to back places them: the id gather
// when count * sparse_den <= n (few rows: read only their sectors), else the
// streaming compaction (read each column once, in order).
struct GatherSpec {
  int m;
  int32_t elem_bytes[RA_MAX_PAYLOAD];
  const void* col[RA_MAX_PAYLOAD];
  void* out[RA_MAX_PAYLOAD];
  int64_t n;           // rows of the relation
  int32_t sparse_den;  // see above (0: the gather always runs)
};
// Gather of payload fields at row ids (the gather stage of a tuple SELECT):
// out_j[i] = col_j[ids[i]] for i < min(*d_count, cap).
int launch_gather(const uint32_t* ids, const int64_t* d_count, int64_t cap, const GatherSpec& g, cudaStream_t s);
// Sparse path without caller ids: the row ids from the select pass's SelMasks
// (exits on the device when the count is dense).
int launch_ids_from_masks(const int32_t* d_key, int64_t n, const SelMasks& mk, const int64_t* d_count,
                          int32_t sparse_den, int64_t staged, uint32_t* ids, cudaStream_t s);
// Payload compaction from the select pass's SelMasks (compact.cu).
int launch_compact(const int32_t* d_key, int64_t n, const SelMasks& mk, const int64_t* d_count, int64_t cap,
                   const GatherSpec& g, cudaStream_t s);

// Fused or unfused chain (validated arguments); used by the C-ABI and fission.
int select_chain_impl(const int32_t* d_in, int64_t n, const ra_pred* h_preds, int k, int fused,
                      int32_t* d_out, int64_t out_cap, int64_t* d_count, void* d_ws,
                      size_t ws_bytes, cudaStream_t s);

// --------------------------------------------------------------- Q1
// accumulate != 0: add into *d_partial (which must hold a valid partial) instead
// of overwriting it — chunks of one query under fission.
int launch_q1(const ra_lineitem& cols, int64_t n, int32_t cutoff, ra_q1_partial* d_partial,
              void* d_ws, size_t ws_bytes, cudaStream_t s, int accumulate = 0);
size_t q1_ws_bytes();
// Leading bytes of a Q1 workspace that carry state between launches (ticket,
// status, grid accumulators): zero them to start a workspace afresh.
size_t q1_ws_clear_bytes();
// Narrow Q1 (f4): same workspace and partial as launch_q1; columns 16-B aligned.
int launch_q1_narrow(const ra_lineitem_narrow& cols, int64_t n, int32_t cutoff, ra_q1_partial* d_partial,
                     void* d_ws, cudaStream_t s, int accumulate = 0);
int launch_q1_encode(const ra_lineitem& in, int64_t n, const ra_lineitem_narrow_out& out, uint32_t* d_status,
                     cudaStream_t s);

}  // namespace ra

// ------------------------------------------------------ device helpers
namespace ra {
namespace dev {

__device__ __forceinline__ int4 ld_stream_v4(const int4* p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ int64_t ld_relaxed_s64(const int64_t* p) {
  int64_t v;
  asm volatile("ld.relaxed.gpu.global.s64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// acq_rel fetch-add: orders this CTA's earlier header reads before the ticket.
__device__ __forceinline__ uint32_t atom_add_acq_rel_u32(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}

// ---- programmatic dependent launch: a kernel launched by launch_pdl may start
// while the previous kernel on the stream finishes; it calls grid_dep_wait()
// before its first global-memory access (the previous grid's writes are then
// visible).
__device__ __forceinline__ void grid_dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// ---- mbarrier + bulk-copy (TMA engine) helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// try_wait with a suspend-time hint: a waiting warp sleeps (up to `ns`)
// instead of re-issuing the probe, leaving issue slots to the warps that work.
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity, uint32_t ns) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAITS_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
      "@!p bra WAITS_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity), "r"(ns)
      : "memory");
}

__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ int64_t warp_sum_s64(int64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

}  // namespace dev
}  // namespace ra
