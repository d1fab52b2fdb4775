// q1_common.cuh — pieces shared by the Q1 kernels of libra.so (wide
// q1_fused.cu and narrow q1_narrow.cu): the per-thread sums, the warp -> CTA
// -> last-CTA 128-bit reduction and the per-CTA partial layout.  Product side
// only (the oracle shares none of this).
#pragma once

#include "ra_internal.cuh"

namespace ra {
namespace q1c {

constexpr int NS = RA_Q1_GROUPS;
constexpr int Q1_MAX_GRID = 148 * 8;

struct Q1Block {  // (sizes the ABI's Q1 workspace: ra_q1_workspace_bytes)
  uint32_t status;
  uint32_t _pad;
  uint64_t v[NS][8];  // count, qty, price, disc, dp_lo, dp_hi, ch_lo, ch_hi
};

// Final per-thread sums handed to the reduction.
struct Acc {
  uint32_t cnt[NS];
  uint32_t sdisc[NS];
  uint64_t sq[NS], sp[NS], sdp[NS], sch[NS];
  uint32_t status;
};

__device__ __forceinline__ void acc_zero(Acc& A) {
#pragma unroll
  for (int s = 0; s < NS; ++s) {
    A.cnt[s] = 0;
    A.sdisc[s] = 0;
    A.sq[s] = A.sp[s] = A.sdp[s] = A.sch[s] = 0;
  }
  A.status = 0;
}

__device__ __forceinline__ void add128(uint64_t& lo, uint64_t& hi, uint64_t lo2, uint64_t hi2) {
  const uint64_t l = lo + lo2;
  hi += hi2 + (l < lo ? 1ull : 0ull);
  lo = l;
}

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ void warp_sum_u128(uint64_t& lo, uint64_t& hi) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t l2 = __shfl_xor_sync(0xffffffffu, lo, o);
    const uint64_t h2 = __shfl_xor_sync(0xffffffffu, hi, o);
    add128(lo, hi, l2, h2);
  }
}

// Grid accumulators (in the workspace; zero between launches): per slot
// ACC_K u64 — count, qty, price, disc, then the 128-bit disc_price and charge
// sums as three limbs each (bits 0-31, bits 32-63, bits 64-127 of every CTA's
// value).  Every CTA adds its partial with 64-bit atomics (RED), so no add
// overflows: <= Q1_MAX_GRID 32-bit limbs sum below 2^43, and the 64-bit
// fields' grid sums stay < 2^63 through SF100 (C11).  The last CTA in reads
// and clears them in ONE round of atomic exchanges and composes the
// ra_q1_partial: a walk over per-CTA partials cost ~6 us of dependent L2
// round trips at the end of every launch (stamped with %globaltimer,
// scripts/q1n_times.py).  Workspace header: u32 CTA ticket @0, u32 status @4.
constexpr int ACC_K = 10;
constexpr int ACC_OFFSET = 256;  // bytes from the workspace start

template <typename Params>
__device__ __forceinline__ void acc_add(const Params& P, int s, int k, uint64_t v) {
  if (v) atomicAdd(P.acc + s * ACC_K + k, (unsigned long long)v);  // result unused: RED
}
// which: 0 = disc_price, 1 = charge
template <typename Params>
__device__ __forceinline__ void acc_add128(const Params& P, int s, int which, uint64_t lo, uint64_t hi) {
  acc_add(P, s, 4 + 3 * which, lo & 0xFFFFFFFFull);
  acc_add(P, s, 5 + 3 * which, lo >> 32);
  acc_add(P, s, 6 + 3 * which, hi);
}

template <typename Params>
__device__ __forceinline__ void publish_and_fold(const Params& P, bool* s_last);

// Reduction: warp (shuffles) -> CTA (smem) -> grid (atomic accumulators, last
// CTA composes).  Called by every thread of the CTA; warps >= NW (a producer
// warp) only join the barriers.  s_w: [NW][NS][8] shared scratch.
template <int NW, typename Params>
__device__ __forceinline__ void reduce_and_fold(const Acc& A, const Params& P, uint64_t (*s_w)[NS][8],
                                                uint32_t* s_status, bool* s_last) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) *s_status = 0;
  __syncthreads();
  if (warp < NW) {
    if (A.status) atomicOr(s_status, A.status);
#pragma unroll
    for (int s = 0; s < NS; ++s) {
      const uint64_t c = warp_sum_u64(A.cnt[s]);
      const uint64_t q = warp_sum_u64(A.sq[s]);
      const uint64_t p = warp_sum_u64(A.sp[s]);
      const uint64_t d = warp_sum_u64(A.sdisc[s]);
      uint64_t dlo = A.sdp[s], dhi = 0, clo = A.sch[s], chi = 0;
      warp_sum_u128(dlo, dhi);
      warp_sum_u128(clo, chi);
      if (lane == 0) {
        s_w[warp][s][0] = c;
        s_w[warp][s][1] = q;
        s_w[warp][s][2] = p;
        s_w[warp][s][3] = d;
        s_w[warp][s][4] = dlo;
        s_w[warp][s][5] = dhi;
        s_w[warp][s][6] = clo;
        s_w[warp][s][7] = chi;
      }
    }
  }
  __syncthreads();
  if (threadIdx.x < NS * 4) {  // (slot, field pair)
    const int s = threadIdx.x >> 2, f = threadIdx.x & 3;
    if (f < 2) {  // count/qty or price/disc: 64-bit
      uint64_t a = 0, b = 0;
      for (int w = 0; w < NW; ++w) {
        a += s_w[w][s][2 * f];
        b += s_w[w][s][2 * f + 1];
      }
      acc_add(P, s, 2 * f, a);
      acc_add(P, s, 2 * f + 1, b);
    } else {  // dp or ch: 128-bit
      uint64_t lo = 0, hi = 0;
      for (int w = 0; w < NW; ++w) add128(lo, hi, s_w[w][s][2 * f], s_w[w][s][2 * f + 1]);
      acc_add128(P, s, f - 2, lo, hi);
    }
  }
  if (threadIdx.x == 0 && *s_status) atomicOr(P.counter + 1, *s_status);
  publish_and_fold(P, s_last);
}

// After this CTA added its partial: ticket; the last CTA to arrive reads and
// clears the accumulators and writes *P.out (128-bit where needed).  Called
// by every thread (blockDim.x > NS * ACC_K).
template <typename Params>
__device__ __forceinline__ void publish_and_fold(const Params& P, bool* s_last) {
  __shared__ unsigned long long s_acc[NS * ACC_K];
  __shared__ uint32_t s_st;
  __threadfence();  // this thread's accumulator adds happen before the ticket
  __syncthreads();
  if (threadIdx.x == 0) *s_last = (atomicAdd(P.counter, 1u) == gridDim.x - 1);
  __syncthreads();
  if (!*s_last) return;

  // ---- last CTA: every other CTA's adds are performed; read + clear at once
  __threadfence();
  if (threadIdx.x < NS * ACC_K) s_acc[threadIdx.x] = atomicExch(P.acc + threadIdx.x, 0ull);
  if (threadIdx.x == NS * ACC_K) s_st = atomicExch(P.counter + 1, 0u);
  __syncthreads();
  if (threadIdx.x < NS * 4) {
    const int s = threadIdx.x >> 2, f = threadIdx.x & 3;
    const unsigned long long* v = s_acc + s * ACC_K;
    uint64_t a, b;
    if (f < 2) {
      a = v[2 * f];
      b = v[2 * f + 1];
    } else {  // limbs (bits 0-31, 32-63, 64-127) -> 128-bit
      const unsigned long long* l = v + 4 + 3 * (f - 2);
      a = l[0];
      b = l[2];
      add128(a, b, l[1] << 32, l[1] >> 32);
    }
    ra_q1_group* G = &P.out->group[s];
    if (P.accumulate) {  // exact: 64-bit sums stay < 2^63 through SF100 (C11), 128-bit ones carry
      const uint64_t* o = reinterpret_cast<const uint64_t*>(G);
      if (f < 2) {
        a += o[2 * f];
        b += o[2 * f + 1];
      } else {
        add128(a, b, o[2 * f], o[2 * f + 1]);
      }
    }
    if (f == 0) {
      G->count = (int64_t)a;
      G->sum_qty = (int64_t)b;
    } else if (f == 1) {
      G->sum_base_price = (int64_t)a;
      G->sum_disc = (int64_t)b;
    } else if (f == 2) {
      G->sum_disc_price_lo = a;
      G->sum_disc_price_hi = (int64_t)b;
    } else {
      G->sum_charge_lo = a;
      G->sum_charge_hi = (int64_t)b;
    }
  } else if (threadIdx.x == NS * 4) {
    const uint32_t st = s_st;
    P.out->status = P.accumulate ? (P.out->status | st) : st;
    P.out->n_groups = NS;
    P.out->rows = P.accumulate ? P.out->rows + (uint64_t)P.n : (uint64_t)P.n;
    *P.counter = 0u;  // self-cleaning for the next launch
  }
}

}  // namespace q1c
}  // namespace ra
