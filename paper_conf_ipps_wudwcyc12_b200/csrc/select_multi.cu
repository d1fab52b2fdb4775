// select_multi.cu — SELECT as one warp-specialised pass for sm_100a: the
// fused chain (one output) and several SELECTs filtering the same input
// ("different SELECT operators need to filter the same input
// data", Fig 2(c)).  Output o is the order-preserving
// SELECT of the input by predicate chain o, o < M <= RA_MAX_OUTPUTS (4).
//
// The input is read once; every output has its own compaction and its own
// global offsets.  The paper's four stages (partition, filter, buffer, gather;
// Fig 3) are split over specialised warps of one
// persistent 768-thread CTA per SM:
//
//   producer warp    draws tiles by atomic ticket, bulk-copies each 32 KB tile
//                    (TMA engine) into a ring of input slots
//   2 compute groups 8 warps each, alternate tiles: filter (all M folded
//                    predicates in registers), per-output warp counts, publish
//                    the M tile aggregates at once, allocate the tile's runs in
//                    a shared ring of selected rows (in tile order), compact
//                    each output's matches into its run
//   3 look-back warps decoupled look-back over the published aggregates: warp
//                    r resolves tiles r, r+3, ... (bulk-copied windows of status
//                    words, branch-free sums), prefixes chained in shared memory
//   4 writer warps   copy each placed tile's M runs from the ring to the
//                    outputs, in tile order, with coalesced stores
//
// The compute path never waits for a placement (an L2 round trip under load)
// except when the ring is full, and then only for OLDER tiles: the ring always
// holds a whole tile's M runs.  setmaxnreg gives the compute warpgroups 88
// registers and the latency-bound aux warpgroups 56.  Tiles are 8192 rows.
// Status words: W = ceil(M/2) u64 words per tile, each [flag:2 | 28-bit launch
// tag | two 16-bit aggregates]; a word is ready when its high half carries this
// launch's tag, so no per-call memset (the launch before the tag wraps clears
// every status word the workspace has carried).  How this design was measured
// into shape (round 1's compute-warp writes and global spills, one look-back
// warp, branchy window sums): DESIGN.md §7.

#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "ra_internal.cuh"

#ifdef RA_MO_TIMES  // diagnostics build: per-CTA %globaltimer stamps (scripts/mo_times.py)
__device__ unsigned long long g_mo_t[2048][16];
#define MO_T(k)                                              \
  do {                                                       \
    unsigned long long t_;                                   \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));   \
    g_mo_t[blockIdx.x][k] = t_;                              \
  } while (0)
extern "C" __attribute__((visibility("default"))) int ramo_times(unsigned long long* out) {
  cudaDeviceSynchronize();
  return (int)cudaMemcpyFromSymbol(out, g_mo_t, sizeof(g_mo_t));
}
#else
#define MO_T(k)
#endif

namespace ra {

namespace {

constexpr uint64_t FLAG_A = 1ull << 62;
constexpr int TAG_SHIFT = 34;
constexpr uint64_t TAG_MASK = (1ull << 28) - 1;
// header: u32 epoch @0, u64 ticket @8, u32 done @16, u64 status-word high-water mark @24
constexpr int H_EPOCH = 0, H_DONE = 4, H_HWM = 6;

#ifndef RA_MO_NG
#define RA_MO_NG 2  // compute groups per CTA
#endif
#ifndef RA_MO_NWR
#define RA_MO_NWR 4  // writer warps per CTA (aux warps fill whole warpgroups)
#endif
#ifndef RA_MO_NWR34
#define RA_MO_NWR34 RA_MO_NWR  // M = 3, 4 (their dense passes are writer-bound)
#define RA_MO_REGS34 RA_MO_REGS
#define RA_MO_AUXREGS34 RA_MO_AUXREGS
#endif
#ifndef RA_MO_REGS
// setmaxnreg: the compute warpgroups run with RA_MO_REGS registers, the aux
// warpgroups (look-back, producer, writers) with RA_MO_AUXREGS; an increase is
// served only from what this CTA's decreases released (0: no rebalancing)
#define RA_MO_REGS 88
#define RA_MO_AUXREGS 56
#endif
#ifndef RA_MO_SCAT_ARRIVALS
// arrivals per tile on `scattered`: every compute thread releases its own ring
// writes (the form compute-sanitizer's racecheck models; one warp-wide arrive
// per warp, measured the same speed as lane 0 after __syncwarp, =GW)
#define RA_MO_SCAT_ARRIVALS GT
#endif
#ifndef RA_MO_WU
#define RA_MO_WU 8  // writer: ring loads in flight per lane
#endif
#ifndef RA_MO_D1
// window of tile k copied once tile k+D1 is counted (or on demand); measured
// best: 2 for one output (the words before a tile are older), 1 for several
// (dense runs wait for the ring sooner)
#define RA_MO_D1 0
#endif
#ifndef RA_MO_IN_KB
#define RA_MO_IN_KB 96  // input ring per CTA, one output
#endif
#ifndef RA_MO_IN_KB2
// two outputs: 2 input slots, the rest of shared memory to the ring of
// selected rows (3 slots were 15% slower when both outputs keep ~half the rows
// with overlapping predicates: the ring filled and placements queued behind it)
#define RA_MO_IN_KB2 64
#endif
constexpr int NG = RA_MO_NG;
constexpr int GW = 8;                         // warps per compute group
constexpr int GT = 32 * GW;                   // threads per compute group
constexpr int NCW = NG * GW;                  // compute warps
#ifndef RA_MO_NLB
#define RA_MO_NLB 3  // look-back warps
#endif
constexpr int NLB = RA_MO_NLB;
constexpr int LBWARP = NCW, PRWARP = NCW + NLB, WR0 = NCW + NLB + 1;
#ifndef RA_MO_K
#define RA_MO_K 8
#endif
constexpr int K = RA_MO_K;                    // metadata slots: tiles counted but not yet written
constexpr int LBW = 10;                       // status words per look-back lane per pass
constexpr int PASS_WORDS = 32 * LBW;
constexpr int Q = NLB;                        // window slots: one per look-back warp
constexpr int WIN_WORDS = 512;                // window slot (status words)
constexpr int SMEM_BUDGET = 232448;           // max dynamic shared memory per CTA on sm_100


#ifndef RA_MO_VEC34
#define RA_MO_VEC34 8     // M = 3, 4: int4 vectors per compute lane per tile
#endif
#ifndef RA_MO_IN_KB34
#define RA_MO_IN_KB34 64  // M = 3, 4: input ring per CTA
#endif
template <int M>
struct Cfg {
  static constexpr int VEC = M <= 2 ? 8 : RA_MO_VEC34;  // int4 vectors per compute lane per tile
  static constexpr int TILE = GT * VEC * 4;          // rows per tile: 8192 | 4096
  static constexpr int WROWS = TILE / GW;            // contiguous rows per compute warp
  static constexpr int NPK = VEC / 4;                // packed 8-bit count words per lane per output
  static constexpr int W = (M + 1) / 2;              // status words per tile
  static constexpr int INSLOTS = (M == 1 ? RA_MO_IN_KB : M == 2 ? RA_MO_IN_KB2 : RA_MO_IN_KB34) * 1024 / (TILE * 4);
  static constexpr int D1 = RA_MO_D1 > 0 ? RA_MO_D1 : (M == 1 ? 2 : 1);
  static constexpr int NWR = M <= 2 ? RA_MO_NWR : RA_MO_NWR34;           // writer warps
  static constexpr int BLOCK = 32 * (NCW + NLB + 1 + NWR);
  static constexpr int REGS = M <= 2 ? RA_MO_REGS : RA_MO_REGS34;         // setmaxnreg: compute warps
  static constexpr int AUXREGS = M <= 2 ? RA_MO_AUXREGS : RA_MO_AUXREGS34;  // and aux warps
};
__host__ __device__ constexpr int q_of(int npk, int j) { return npk == 2 ? (j & 1) : 0; }
__host__ __device__ constexpr int b_of(int npk, int j) { return npk == 2 ? (j >> 1) : ((j >> 1) | ((j & 1) << 1)); }

struct MoParams {
  const int32_t* abase;  // 16-B aligned base, = d_in - mis
  int64_t n;             // rows (host bound)
  const int64_t* d_n;    // optional device row count (<= n): the previous pass's count (unfused chain)
  uint32_t* hdr;
  unsigned long long* ticket;
  uint64_t* status;      // status[tile * W + j]
  int32_t mis;
  int32_t lo[RA_MAX_OUTPUTS];
  uint32_t span[RA_MAX_OUTPUTS];
  int32_t n_ne[RA_MAX_OUTPUTS];
  int32_t ne[RA_MAX_OUTPUTS][RA_MAX_PREDS];
  int32_t* out[RA_MAX_OUTPUTS];
  int64_t out_cap[RA_MAX_OUTPUTS];
  int64_t* d_count[RA_MAX_OUTPUTS];
};

template <int M>
struct MoFixed {  // everything but the ring
  int4 in[Cfg<M>::INSLOTS][Cfg<M>::TILE / 4];
  uint64_t win[Q][WIN_WORDS];
  uint64_t full[Cfg<M>::INSLOTS], empty[Cfg<M>::INSLOTS];
  uint64_t winfull[Q];
  uint64_t counted[K], placed[K], scattered[K], written[K], allocd[K];
  int64_t tile_of[Cfg<M>::INSLOTS];
  int64_t tidx[K];
  int64_t goff[K][M];
  int64_t wlo[Q], whi[Q];
  int64_t vstart[K];  // virtual start of the tile's runs (see the allocator)
  int64_t a_va;       // allocator: virtual end of the newest tile's runs (tile order, one thread at a time)
  int32_t w_done;     // writers: tiles written
  int32_t cnt[K][M];
  int32_t start[K];  // ring position of the tile's first run (runs back to back, output order)
  uint32_t wtot[2 * NG][M][GW];
  int64_t pfx[M];     // look-back chain: inclusive prefixes after tile chain_done - 1
  int32_t chain_done; // tiles placed
  int32_t end_tile;   // the CTA's end-marker tile index (INT32_MAX until known)
  int32_t lb_done;    // look-back warps finished
  int64_t n;
  uint32_t epoch;
  int32_t demand;
#ifdef RA_MO_PROFILE
  long long t_count[K], t_placed[K], t_issue[Q];
#endif
};
template <int M>
constexpr int ring_ints() {
  return (int)((SMEM_BUDGET - ((sizeof(MoFixed<M>) + 127) / 128) * 128 - 128) / 4) / 32 * 32;
}
template <int M>
struct __align__(128) MoSmem : MoFixed<M> {
  static constexpr int RING = ring_ints<M>();
  alignas(128) int32_t ring[RING];  // runs start at multiples of 32 rows (128-B aligned)
};
// the producer ends with one marker per compute group in consecutive slots,
// and a group that takes a marker releases no slot: every marker needs its own
static_assert(Cfg<1>::INSLOTS >= NG && Cfg<2>::INSLOTS >= NG && Cfg<3>::INSLOTS >= NG && Cfg<4>::INSLOTS >= NG,
              "input slots >= compute groups");
static_assert(MoSmem<1>::RING >= Cfg<1>::TILE && MoSmem<2>::RING >= 2 * Cfg<2>::TILE &&
                  MoSmem<3>::RING >= 3 * Cfg<3>::TILE && MoSmem<4>::RING >= 4 * Cfg<4>::TILE,
              "a tile's M runs must always fit an empty ring");
static_assert(sizeof(MoSmem<1>) <= SMEM_BUDGET && sizeof(MoSmem<2>) <= SMEM_BUDGET &&
                  sizeof(MoSmem<3>) <= SMEM_BUDGET && sizeof(MoSmem<4>) <= SMEM_BUDGET,
              "shared memory");

using dev::bulk_g2s;
using dev::mbar_arrive;
using dev::mbar_arrive_expect_tx;
using dev::mbar_init;
using dev::mbar_test;
using dev::mbar_wait;
using dev::smem_u32;

#ifdef RA_MO_PROFILE  // diagnostics build: per-wait cycle totals (lane 0 of each waiting warp)
__device__ unsigned long long g_mo_prof[32], g_mo_cnt[32];
#define PROF_T0(v) const long long v = clock64()
#define PROF_STAMP(dst) dst = clock64()
#define PROF_LAT(code, src)              \
  do {                                   \
    const long long t_l_ = src;          \
    PROF_ADD(code, t_l_);                \
  } while (0)
#define PROF_SINCE(code, v) PROF_ADD(code, v)
#define PROF_ADD(code, v)                                               \
  do {                                                                  \
    if ((threadIdx.x & 31) == 0 && blockIdx.x == 0) {                   \
      atomicAdd(&g_mo_prof[code], (unsigned long long)(clock64() - v)); \
      atomicAdd(&g_mo_cnt[code], 1ull);                                 \
    }                                                                   \
  } while (0)
#define MWAIT(bar, parity, code, idx) \
  do {                                \
    PROF_T0(t_w_);                    \
    mbar_wait(bar, parity);           \
    PROF_ADD(code, t_w_);             \
  } while (0)
#else
#define PROF_T0(v)
#define PROF_ADD(code, v)
#define PROF_STAMP(dst)
#define PROF_LAT(code, src)
#endif

#if defined(RA_MO_PROFILE)
#elif defined(RA_MO_WATCHDOG)  // diagnostics build: a wait that exceeds ~4 s reports itself and traps
__device__ __noinline__ void mwait(uint64_t* bar, uint32_t parity, int code, int idx) {
  const long long t0 = clock64();
  while (!mbar_test(bar, parity)) {
    if (clock64() - t0 > 8000000000ll) {
      printf("select_multi watchdog: block %d warp %d lane %d wait %d idx %d parity %u\n", (int)blockIdx.x,
             (int)(threadIdx.x >> 5), (int)(threadIdx.x & 31), code, idx, parity);
      __trap();
    }
  }
}
#define MWAIT(bar, parity, code, idx) mwait(bar, parity, code, idx)
#else
#define MWAIT(bar, parity, code, idx) mbar_wait(bar, parity)
#endif

__device__ __forceinline__ void st_relaxed_shared(int32_t* p, int32_t v) {
  asm volatile("st.relaxed.cta.shared.b32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}
__device__ __forceinline__ int32_t ld_relaxed_shared(const int32_t* p) {
  int32_t v;
  asm volatile("ld.relaxed.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ int32_t ld_acquire_shared(const int32_t* p) {
  int32_t v;
  asm volatile("ld.acquire.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_shared(int32_t* p, int32_t v) {
  asm volatile("st.release.cta.shared.b32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void group_bar(int g) {  // named barriers 1..NG: one compute group
  asm volatile("bar.sync %0, %1;" ::"r"(1 + g), "n"(GT) : "memory");
}
template <int NWR>
__device__ __forceinline__ void writer_bar() {
  asm volatile("bar.sync %0, %1;" ::"n"(1 + NG), "n"(32 * NWR) : "memory");
}
// st.shared v at byte address a and advance a, iff (fl & mask) != 0 (one
// predicated store + add per row; see select_fused.cu)
__device__ __forceinline__ void put_if(uint32_t& a, uint32_t fl, uint32_t mask, int32_t v) {
  asm volatile(
      "{\n\t.reg .pred q;\n\t.reg .b32 t;\n\t"
      "and.b32 t, %1, %2;\n\t"
      "setp.ne.u32 q, t, 0;\n\t"
      "@q st.shared.b32 [%0], %3;\n\t"
      "@q add.u32 %0, %0, 4;\n\t}"
      : "+r"(a)
      : "r"(fl), "r"(mask), "r"(v)
      : "memory");
}
__device__ __forceinline__ int32_t comp(const int4& v, int c) { return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w; }

template <bool HAS_NE>
__device__ __forceinline__ bool keep(int32_t x, const MoParams& P, int o) {
  bool k = (uint32_t)x - (uint32_t)P.lo[o] <= P.span[o];  // lo <= x <= hi (mod-2^32 difference)
  if (HAS_NE) {
#pragma unroll
    for (int j = 0; j < RA_MAX_PREDS; ++j)
      if (j < P.n_ne[o]) k &= (x != P.ne[o][j]);
  }
  return k;
}

// Look-back lane 0: bulk-copy the status words of tiles [lo, hi) into window
// slot q (a window longer than the slot is read directly instead).
template <int M>
__device__ __forceinline__ void issue_window(MoSmem<M>& S, const MoParams& P, int q, int64_t lo, int64_t hi) {
  constexpr int W = Cfg<M>::W;
  S.wlo[q] = lo;
  S.whi[q] = hi;
  const int64_t w0 = lo * W, w1 = hi * W, s0 = w0 & ~1ll;
  if (w1 <= w0 || w1 - s0 > WIN_WORDS) {
    mbar_arrive(&S.winfull[q]);
    return;
  }
  const uint32_t bytes = (uint32_t)(((w1 - s0) * 8 + 15) & ~15ll);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_arrive_expect_tx(&S.winfull[q], bytes);
  bulk_g2s(&S.win[q][0], P.status + s0, bytes, &S.winfull[q]);
}

// Per-output sums of the aggregates of tiles [wlo, whi) (one warp).  Lane l
// takes words base + l + 32c (conflict-free shared loads; with W = 2 words per
// tile a lane's words all carry the same output pair, l & 1).  A word of this
// launch has high half == want; unpublished words are re-polled from global
// memory.  Branch-free on the copied fast path (clamped addresses + selects).
template <int M>
__device__ __forceinline__ void window_sums(const MoSmem<M>& S, const MoParams& P, int q, int lane, uint32_t want,
                                            int64_t (&t)[M]) {
  constexpr int W = Cfg<M>::W;
  const int64_t w0 = S.wlo[q] * W, w1 = S.whi[q] * W, s0 = w0 & ~1ll;
  const bool copied = w1 > w0 && w1 - s0 <= WIN_WORDS;
  const uint64_t pad = (uint64_t)want << 32;  // a ready word with zero aggregates
#pragma unroll
  for (int o = 0; o < M; ++o) t[o] = 0;
  for (int64_t base = w0 & ~1ll; base < w1; base += PASS_WORDS) {  // even base: word parity = lane parity
    uint64_t w[LBW];
    if (copied) {
#pragma unroll
      for (int c = 0; c < LBW; ++c) {
        const int64_t idx = base + lane + 32 * c;
        const bool in = idx >= w0 && idx < w1;
        const uint64_t x = S.win[q][(in ? idx : w0) - s0];
        w[c] = in ? x : pad;
      }
    } else {
#pragma unroll
      for (int c = 0; c < LBW; ++c) {
        const int64_t idx = base + lane + 32 * c;
        w[c] = (idx >= w0 && idx < w1) ? dev::ld_relaxed_u64(P.status + idx) : pad;
      }
    }
    for (int spins = 0;; ++spins) {
      bool missing = false;
#pragma unroll
      for (int c = 0; c < LBW; ++c) missing |= (uint32_t)(w[c] >> 32) != want;
#ifdef RA_MO_PROFILE
      if (lane == 0 && blockIdx.x == 0) {
        if (spins == 0) atomicAdd(&g_mo_prof[22], (unsigned long long)(w1 - w0));
        if (spins == 0) atomicAdd(&g_mo_cnt[22], 1ull);
        if (spins == 0 && !copied) atomicAdd(&g_mo_prof[23], 1ull);
        if (spins == 0) atomicAdd(&g_mo_cnt[23], 1ull);
      }
#endif
      if (!__any_sync(0xffffffffu, missing)) break;
#ifdef RA_MO_PROFILE
      if (lane == 0 && blockIdx.x == 0) atomicAdd(&g_mo_prof[24], 1ull);
#endif
      if (spins > 1) __nanosleep(64);
#ifdef RA_MO_WATCHDOG
      if (spins == 20000000) {
        for (int c = 0; c < LBW; ++c)
          if ((uint32_t)(w[c] >> 32) != want)
            printf("select_multi watchdog: block %d window word %lld = %llx want %x\n", (int)blockIdx.x,
                   (long long)(base + lane + 32 * c), (unsigned long long)w[c], want);
        __trap();
      }
#endif
#pragma unroll
      for (int c = 0; c < LBW; ++c)
        if ((uint32_t)(w[c] >> 32) != want) w[c] = dev::ld_relaxed_u64(P.status + base + lane + 32 * c);
    }
    uint32_t lo16 = 0, hi16 = 0;  // this lane's two fields (output pair lane & 1 when W == 2)
#pragma unroll
    for (int c = 0; c < LBW; ++c) {
      lo16 += (uint32_t)w[c] & 0xFFFFu;
      hi16 += ((uint32_t)w[c] >> 16) & 0xFFFFu;
    }
#pragma unroll
    for (int o = 0; o < M; ++o) {
      const bool mine = W == 1 || (lane & 1) == (o >> 1);
      t[o] += __reduce_add_sync(0xffffffffu, mine ? ((o & 1) ? hi16 : lo16) : 0u);
    }
  }
}

template <int M, bool HAS_NE>
__global__ void __launch_bounds__(Cfg<M>::BLOCK, 1) select_multi_kernel(const __grid_constant__ MoParams P) {
  using C = Cfg<M>;
  using SM = MoSmem<M>;
  constexpr int TILE = C::TILE, VEC = C::VEC, NPK = C::NPK, W = C::W, INSLOTS = C::INSLOTS, D1 = C::D1;
  constexpr int RING = SM::RING;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  SM& S = *reinterpret_cast<SM*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  if (tid == 0) MO_T(0);
  dev::grid_dep_wait();  // programmatic dependent launch: previous grid's writes visible
  if (tid == 0) {
    MO_T(1);
#ifdef RA_MO_TIMES
    unsigned smid_;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid_));
    g_mo_t[blockIdx.x][8] = smid_;
#endif
    int64_t n = P.n;
    if (P.d_n) {
      const int64_t dn = dev::ld_relaxed_s64(P.d_n);
      n = dn < n ? (dn < 0 ? 0 : dn) : n;
    }
    S.n = n;
    S.epoch = ld_acquire_u32(&P.hdr[H_EPOCH]);
    S.demand = -1;
    S.a_va = 0;
    S.w_done = 0;
    S.chain_done = 0;
    S.end_tile = 0x7fffffff;
    S.lb_done = 0;
    for (int o = 0; o < M; ++o) S.pfx[o] = 0;
  }
  // mbarriers initialised in parallel, one thread each (a serial init by one
  // thread was ~0.5 us of every launch's ramp)
  static_assert(2 * INSLOTS <= 32 && Q <= 32 && K <= 32, "init lanes");
  if (tid >= 32 && tid < 32 + 2 * INSLOTS) mbar_init(tid & 1 ? &S.empty[(tid - 32) >> 1] : &S.full[(tid - 32) >> 1], 1);
  if (tid >= 64 && tid < 64 + Q) mbar_init(&S.winfull[tid - 64], 1);
  if (tid >= 96 && tid < 96 + K) {
    const int s = tid - 96;
    mbar_init(&S.counted[s], 1);
    mbar_init(&S.placed[s], 1);
    mbar_init(&S.scattered[s], RA_MO_SCAT_ARRIVALS);
    mbar_init(&S.written[s], 1);
    mbar_init(&S.allocd[s], 1);
  }
  if ((tid >= 32 && tid < 32 + 2 * INSLOTS) || (tid >= 64 && tid < 64 + Q) || (tid >= 96 && tid < 96 + K))
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
#ifndef RA_MO_LATE_TICKET
#define RA_MO_LATE_TICKET 0
#endif
  // the producer's first ticket is drawn before the barrier: its round trip
  // overlaps the init (the previous launch reset the ticket; grid_dep_wait above)
  int64_t first_ticket = 0;
  if (!RA_MO_LATE_TICKET && warp == PRWARP && lane == 0) first_ticket = (int64_t)atomicAdd(P.ticket, 1ull);
  __syncthreads();
  if (tid == 0) MO_T(2);
  const int64_t n = S.n;
  const int64_t nv = n + P.mis;
  const int64_t ntiles = n > 0 ? (nv + TILE - 1) / TILE : 0;
  const uint64_t tag = S.epoch & TAG_MASK;

  // Aux warps (producer, look-back, writers) first; with RA_MO_REGS the
  // register file is rebalanced: compute warpgroups get more registers, the
  // latency-bound aux warpgroups fewer (setmaxnreg, whole warpgroups).
#if RA_MO_REGS
  static_assert(NCW % 4 == 0 && (C::BLOCK / 32) % 4 == 0, "setmaxnreg works on whole warpgroups");
  if (warp >= NCW) asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(C::AUXREGS));
#endif
  if (warp == PRWARP) {
    // ========================= producer: partition + load =====================
    if (lane == 0) {
      int64_t cur = first_ticket;
      int ends = 0;
      for (int j = 0;; ++j) {
        const int s = j % INSLOTS;
        if (j >= INSLOTS) MWAIT(&S.empty[s], (uint32_t)((j / INSLOTS - 1) & 1), 1, (int)j);
        if (RA_MO_LATE_TICKET && ends == 0) cur = (int64_t)atomicAdd(P.ticket, 1ull);
        if (cur >= ntiles) {  // one end marker per compute group (ntiles + e: e = 0 is the true end)
          if (ends == 0) MO_T(3);
          S.tile_of[s] = ntiles + ends;
          mbar_arrive(&S.full[s]);
          if (++ends == NG) break;
          continue;
        }
        S.tile_of[s] = cur;
        const int64_t v0 = cur * TILE;
        int64_t rows = nv - v0;
        if (rows > TILE) rows = TILE;
        const uint32_t bytes = (uint32_t)((rows * 4 + 15) & ~15ll);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_arrive_expect_tx(&S.full[s], bytes);
        bulk_g2s(&S.in[s][0], P.abase + v0, bytes, &S.full[s]);
        if (!RA_MO_LATE_TICKET) cur = (int64_t)atomicAdd(P.ticket, 1ull);  // next ticket overlaps this copy
      }
    }
    return;
  }

  if (warp >= LBWARP && warp < LBWARP + NLB) {
    // ========================= look-back: tile offsets ========================
    // NLB warps; warp r resolves the CTA's tiles k = r, r + NLB, ...: its
    // window (the tiles strictly between tile k-1 and tile k of this CTA) is
    // bulk-copied into the warp's own window slot once tile k+D1 is counted
    // (its predecessors' words are then almost surely published) or at once
    // on demand (the ring is full), and summed; the sums of consecutive tiles
    // then chain through shared memory (pfx, chain_done): a few instructions.
    // The windows of NLB tiles are in flight and summed in parallel.
    const int r = warp - LBWARP;
    const uint32_t want = (uint32_t)((FLAG_A | (tag << TAG_SHIFT)) >> 32);
#ifdef RA_MO_WATCHDOG
    long long t_wd = clock64();
#endif
    for (int k = r;; k += NLB) {
      // tile k counted, or k is past the CTA's end marker (end_tile < k: done)
      bool past = false;
      for (int spins = 0;; ++spins) {
        if (__all_sync(0xffffffffu, mbar_test(&S.counted[k % K], (uint32_t)((k / K) & 1)))) break;
        if (__all_sync(0xffffffffu, ld_acquire_shared(&S.end_tile) < k)) {
          past = true;
          break;
        }
        if (spins > 2) __nanosleep(32);
#ifdef RA_MO_WATCHDOG
        if (spins == 40000000 && lane == 0) {
          printf("select_multi watchdog: block %d look-back %d counted k %d end %d\n", (int)blockIdx.x, r, k, S.end_tile);
          __trap();
        }
#endif
      }
      if (past) break;
      const int64_t tc = S.tidx[k % K];
      if (tc < 0) {  // end marker (tile k == the CTA's tile count): tell the writers after every placement
        if (lane == 0) {
          while (ld_acquire_shared(&S.chain_done) != k) {}
          mbar_arrive(&S.placed[k % K]);
        }
        break;
      }
      int64_t tprev = -1;
      if (k > 0) {
        MWAIT(&S.counted[(k - 1) % K], (uint32_t)(((k - 1) / K) & 1), 2, k - 1);
        tprev = S.tidx[(k - 1) % K];
      }
      // due: tile k+D1 counted (or the end marker), or the ring waits for tile k
      for (int spins = 0;; ++spins) {
        if (__all_sync(0xffffffffu, ld_relaxed_shared(&S.demand) >= k)) break;
        if (__all_sync(0xffffffffu, mbar_test(&S.counted[(k + D1) % K], (uint32_t)(((k + D1) / K) & 1)))) break;
        if (__all_sync(0xffffffffu, ld_acquire_shared(&S.end_tile) <= k + D1)) break;
        if (spins > 2) __nanosleep(32);
#ifdef RA_MO_WATCHDOG
        if (spins == 40000000 && lane == 0) {
          printf("select_multi watchdog: block %d look-back %d due k %d demand %d\n", (int)blockIdx.x, r, k, S.demand);
          __trap();
        }
#endif
      }
      if (lane == 0) {
        issue_window(S, P, r, tprev + 1, tc);
        PROF_STAMP(S.t_issue[r]);
        PROF_LAT(21, S.t_count[k % K]);
      }
      MWAIT(&S.winfull[r], (uint32_t)((k / NLB) & 1), 3, k);
      if (lane == 0) PROF_LAT(20, S.t_issue[r]);
      int64_t ws[M];
      PROF_T0(t_ws);
      window_sums<M>(S, P, r, lane, want, ws);
      PROF_ADD(17, t_ws);
      __syncwarp();
      if (lane == 0) {
        while (ld_acquire_shared(&S.chain_done) != k) {}  // tile k-1 placed: its prefix is in pfx
#pragma unroll
        for (int o = 0; o < M; ++o) {
          const int64_t g = S.pfx[o] + ws[o];
          S.goff[k % K][o] = g;
          S.pfx[o] = g + S.cnt[k % K][o];
        }
        if (tc == ntiles - 1) {  // the last tile: every tile has published; the totals
#pragma unroll
          for (int o = 0; o < M; ++o) *P.d_count[o] = S.pfx[o];
        }
        PROF_LAT(18, S.t_count[k % K]);
        PROF_STAMP(S.t_placed[k % K]);
        st_release_shared(&S.chain_done, k + 1);
        mbar_arrive(&S.placed[k % K]);
      }
      __syncwarp();
    }
    // the CTA's last look-back warp out joins the grid-wide epilogue: the last
    // CTA out resets the ticket, at a tag wrap clears every status word, and
    // advances the epoch — after every CTA of this launch read it, so all of
    // them (also a late one that drew no tile) used the same tag
    if (lane == 0 && atomicAdd(&S.lb_done, 1) == NLB - 1) {
      MO_T(6);
      __threadfence();
      if (atomicAdd(&P.hdr[H_DONE], 1u) == gridDim.x - 1) {
        *P.ticket = 0ull;
        P.hdr[H_DONE] = 0u;
        if (ntiles == 0) {
#pragma unroll
          for (int o = 0; o < M; ++o) *P.d_count[o] = 0;
        }
        uint64_t* hwm = reinterpret_cast<uint64_t*>(P.hdr + H_HWM);
        uint64_t h = *hwm;
        if ((uint64_t)(ntiles * W) > h) *hwm = h = (uint64_t)(ntiles * W);
        if (((S.epoch + 1) & TAG_MASK) == 0)
          for (uint64_t w = 0; w < h; ++w) P.status[w] = 0ull;
        st_release_u32(&P.hdr[H_EPOCH], S.epoch + 1);
      }
    }
    return;
  }

  if (warp >= WR0) {
    // ========================= writers: ring -> outputs =======================
    // NWR writer warps copy each placed tile's runs, in tile order, with
    // coalesced 128-B warp stores and WU ring loads in flight per lane.
    // (TMA bulk tensor stores of the runs — 1-D maps, element coordinates —
    // were measured slower for dense runs: DESIGN.md §7.)
    const int wt = tid - 32 * WR0;
    constexpr int NWR = C::NWR, WT = 32 * NWR, WU = RA_MO_WU;
    for (int k = 0;; ++k) {
      MWAIT(&S.placed[k % K], (uint32_t)((k / K) & 1), 4, (int)k);
      if (S.tidx[k % K] < 0) {
        if (wt == 0) MO_T(7);
        break;
      }
      MWAIT(&S.scattered[k % K], (uint32_t)((k / K) & 1), 5, (int)k);
      int32_t base = S.start[k % K];
      PROF_T0(t_wr);
#pragma unroll
      for (int o = 0; o < M; ++o) {
        const int32_t c = S.cnt[k % K][o];
        const int64_t g = S.goff[k % K][o];
        const int32_t* run = S.ring + base;
        int32_t* __restrict__ out = P.out[o] + g;
        const int64_t cap = P.out_cap[o] - g;  // rows of this run that fit
        const int64_t lim = cap < 0 ? 0 : (cap > c ? c : cap);
        int e = wt;
        for (; e + (WU - 1) * WT < (int)lim; e += WU * WT) {
          int32_t a[WU];
#pragma unroll
          for (int u = 0; u < WU; ++u) a[u] = run[e + u * WT];
#pragma unroll
          for (int u = 0; u < WU; ++u) out[e + u * WT] = a[u];
        }
        for (; e < (int)lim; e += WT) out[e] = run[e];
        base += (c + 31) & ~31;
      }
      writer_bar<NWR>();  // every writer is done reading the ring
      PROF_ADD(16, t_wr);
      if (wt == 0) {
        PROF_LAT(19, S.t_placed[k % K]);
        st_release_shared(&S.w_done, k + 1);  // the ring reads above happen-before a reuse of the space
        mbar_arrive(&S.written[k % K]);  // release: the ring space
      }
    }
    return;
  }

  // ========================= compute groups =====================================
#if RA_MO_REGS
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(C::REGS));
#endif
  const int g = warp / GW, wg = warp % GW, gtid = tid - GT * g;
  for (int i = g;; i += NG) {
    const int slot = i % INSLOTS;
    PROF_T0(t_it);
    MWAIT(&S.full[slot], (uint32_t)((i / INSLOTS) & 1), 6, (int)i);
    if (i == 0 && gtid == 0) MO_T(4);
    const int64_t t = S.tile_of[slot];
    if (t >= ntiles) {
      if (t == ntiles && gtid == 0) {  // the true end: tile i is this CTA's tile count
        MO_T(5);
        if (i >= K) MWAIT(&S.written[i % K], (uint32_t)(((i / K) - 1) & 1), 7, (int)i);
        S.tidx[i % K] = -1;
        st_release_shared(&S.end_tile, i);
        mbar_arrive(&S.counted[i % K]);
      }
      break;
    }
    // ---- filter
    int4 v[VEC];
    {
      const int4* base = &S.in[slot][wg * (C::WROWS / 4)];
#pragma unroll
      for (int j = 0; j < VEC; ++j) v[j] = base[32 * j + lane];
    }
    const int64_t v0 = t * TILE + wg * C::WROWS;
    uint32_t fl[M];  // bit 4j+c: row wg*WROWS + 4*(32j + lane) + c kept by output o
#pragma unroll
    for (int o = 0; o < M; ++o) fl[o] = 0;
    if (v0 >= P.mis && v0 + C::WROWS <= nv) {
#pragma unroll
      for (int j = 0; j < VEC; ++j)
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
          for (int o = 0; o < M; ++o) fl[o] |= (uint32_t)keep<HAS_NE>(comp(v[j], c), P, o) << (4 * j + c);
    } else {
#pragma unroll
      for (int j = 0; j < VEC; ++j) {
        const int64_t e0 = v0 + 4 * (32 * j + lane);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const bool in = (e0 + c >= P.mis) & (e0 + c < nv);
#pragma unroll
          for (int o = 0; o < M; ++o) fl[o] |= (uint32_t)(keep<HAS_NE>(comp(v[j], c), P, o) & in) << (4 * j + c);
        }
      }
    }
    // ---- per-output warp counts -> group totals
    const int wslot = i % (2 * NG);
#pragma unroll
    for (int o = 0; o < M; ++o) {
      const uint32_t wc = __reduce_add_sync(0xffffffffu, (uint32_t)__popc(fl[o]));
      if (lane == 0) S.wtot[wslot][o][wg] = wc;
    }
    PROF_T0(t_b1);
    group_bar(g);  // B1: counts visible; the group is done reading the input slot
    PROF_ADD(12, t_b1);
    int32_t agg[M], wbase[M];
#pragma unroll
    for (int o = 0; o < M; ++o) {
      const uint32_t wt_ = lane < GW ? S.wtot[wslot][o][lane] : 0u;
      agg[o] = (int32_t)__reduce_add_sync(0xffffffffu, wt_);
      wbase[o] = (int32_t)__reduce_add_sync(0xffffffffu, lane < wg ? wt_ : 0u);
    }
    if (gtid == 0) {
      PROF_T0(t_g0);
      mbar_arrive(&S.empty[slot]);  // the producer refills the slot
      if (i >= K) MWAIT(&S.written[i % K], (uint32_t)(((i / K) - 1) & 1), 8, (int)i);  // metadata slot free
      // publish the M aggregates at once (W words, each self-validating)
#pragma unroll
      for (int j = 0; j < W; ++j) {
        const uint64_t a = (uint64_t)(uint32_t)agg[2 * j] | ((2 * j + 1 < M ? (uint64_t)(uint32_t)agg[2 * j + 1] : 0ull) << 16);
        dev::st_relaxed_u64(P.status + t * W + j, FLAG_A | (tag << TAG_SHIFT) | a);
      }
      // (the tile's runs are each padded to a multiple of 32 rows: 128-B aligned starts)
#pragma unroll
      for (int o = 0; o < M; ++o) S.cnt[i % K][o] = agg[o];
      S.tidx[i % K] = t;
      PROF_STAMP(S.t_count[i % K]);
      mbar_arrive(&S.counted[i % K]);
      PROF_ADD(13, t_g0);
    }
    if (gtid == 0) {
      int32_t rows_in = 0;
#pragma unroll
      for (int o = 0; o < M; ++o) rows_in += (agg[o] + 31) & ~31;
      // ---- allocate the tile's runs, in CTA tile order (after tile i-1's).
      // Virtual ring coordinates grow monotonically; a run set that would
      // cross the physical end starts at the next multiple of RING.  Pending
      // (unwritten) rows are [vstart of the oldest unwritten tile, a_va), so
      // the new runs fit once their end is within RING of that start, or at
      // once when every earlier tile is written.  Every tile fits an empty ring.
      if (i > 0) MWAIT(&S.allocd[(i - 1) % K], (uint32_t)(((i - 1) / K) & 1), 9, (int)i);
      int64_t s0 = S.a_va;
      if ((int32_t)(s0 % RING) + rows_in > RING) s0 = (s0 / RING + 1) * RING;
      const int64_t vend = s0 + rows_in;
      while (true) {
        // h = tiles written so far (>= i - K + 1: tile i - K is written)
        const int32_t h = ld_acquire_shared(&S.w_done);
        if (h >= i || vend - S.vstart[h % K] <= RING) break;
        st_relaxed_shared(&S.demand, h);  // the look-back places tile h without delay
        MWAIT(&S.written[h % K], (uint32_t)((h / K) & 1), 10, (int)h);
      }
      S.start[i % K] = (int32_t)(s0 % RING);
      S.vstart[i % K] = s0;
      S.a_va = vend;
      mbar_arrive(&S.allocd[i % K]);
    }
    PROF_T0(t_b2);
    group_bar(g);  // B2: the run start is visible
    PROF_ADD(14, t_b2);
    PROF_T0(t_sc);
    // ---- scatter each output's matches into its run
    int32_t rb = S.start[i % K];
    const uint32_t ring0 = smem_u32(S.ring);
#pragma unroll
    for (int o = 0; o < M; ++o) {
      const uint32_t f = fl[o];
      uint32_t packed[NPK], inc[NPK], tot[NPK];
      uint32_t x = f - ((f >> 1) & 0x55555555u);  // SWAR nibble popcounts: nibble j = vector j's 4 rows
      x = (x & 0x33333333u) + ((x >> 2) & 0x33333333u);
      if (NPK == 2) {
        packed[0] = x & 0x0F0F0F0Fu;
        packed[NPK - 1] = (x >> 4) & 0x0F0F0F0Fu;
      } else {
        packed[0] = (x & 0x0F0Fu) | (((x >> 4) & 0x0F0Fu) << 16);
      }
#pragma unroll
      for (int q = 0; q < NPK; ++q) inc[q] = packed[q];
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
        for (int q = 0; q < NPK; ++q) {
          const uint32_t y = __shfl_up_sync(0xffffffffu, inc[q], d);
          if (lane >= d) inc[q] += y;
        }
      }
#pragma unroll
      for (int q = 0; q < NPK; ++q) tot[q] = __shfl_sync(0xffffffffu, inc[q], 31);
      int32_t r = rb + wbase[o];
#pragma unroll
      for (int j = 0; j < VEC; ++j) {
        const int q = q_of(NPK, j), b = b_of(NPK, j);
        const int32_t p = r + (int32_t)(((inc[q] - packed[q]) >> (8 * b)) & 0xFFu);
        uint32_t a = ring0 + 4u * (uint32_t)p;
#pragma unroll
        for (int c = 0; c < 4; ++c) put_if(a, f, 1u << (4 * j + c), comp(v[j], c));
        r += (int32_t)((tot[q] >> (8 * b)) & 0xFFu);
      }
      rb += (agg[o] + 31) & ~31;
    }
    __syncwarp();
    if (RA_MO_SCAT_ARRIVALS == GT || lane == 0) mbar_arrive(&S.scattered[i % K]);
    PROF_ADD(15, t_sc);
    PROF_ADD(11, t_it);
  }
}

template <int M, bool HAS_NE>
int launch_mo(const MoParams& P, int64_t ntiles, cudaStream_t s) {
  static std::atomic<int> attr[64];
  const int a = device_once(attr, current_device(), [] {
    cudaError_t e = cudaFuncSetAttribute(select_multi_kernel<M, HAS_NE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sizeof(MoSmem<M>));
    return e != cudaSuccess ? cuda_fail(e, "cudaFuncSetAttribute(select_multi smem)") : 1;
  });
  if (a < 0) return a;
  int64_t grid = num_sms();  // persistent: one CTA per SM
  // RA_SEL_MAX_CTAS (diagnostics only): cap the grid, for the paper's Fig 12
  // experiment (a SELECT with half the CTAs, two of them on two streams)
  static const int64_t max_ctas = getenv("RA_SEL_MAX_CTAS") ? atoll(getenv("RA_SEL_MAX_CTAS")) : 0;
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
  if (grid > ntiles) grid = ntiles;
  if (grid < 1) grid = 1;
  cudaError_t e = launch_pdl(select_multi_kernel<M, HAS_NE>, dim3((unsigned)grid), dim3(Cfg<M>::BLOCK), sizeof(MoSmem<M>), s, P);
  count_launch();
  if (e != cudaSuccess) return cuda_fail(e, "select_multi_kernel launch");
  return RA_OK;
}

}  // namespace

int64_t mo_tile_rows(int M) { return M <= 2 ? Cfg<1>::TILE : Cfg<3>::TILE; }
static_assert(Cfg<3>::TILE == Cfg<4>::TILE, "one tile size for M = 3, 4");

size_t mo_workspace_bytes(int64_t n) {
  // worst case over M: the smaller tile (+3 rows of misalignment, +1), two words each
  constexpr int64_t T = Cfg<1>::TILE < Cfg<3>::TILE ? Cfg<1>::TILE : Cfg<3>::TILE;
  const int64_t tiles = (n + 3 + T - 1) / T + 1;
  return ((SEL_HDR_BYTES + 16 * (size_t)tiles + 16) + 255) / 256 * 256;
}


int launch_select_multi(const int32_t* d_in, int64_t n, const CanonPred* cp, int M, int32_t* const* d_outs,
                        const int64_t* out_caps, int64_t* const* d_counts, void* d_ws, cudaStream_t s,
                        const int64_t* d_n) {
  if (M < 1 || M > RA_MAX_OUTPUTS) return fail(RA_E_INVAL, "M=%d outside [1, %d]", M, RA_MAX_OUTPUTS);
  if (n >= ((int64_t)1 << 34)) return fail(RA_E_INVAL, "n=%lld >= 2^34", (long long)n);
  MoParams P;
  memset(&P, 0, sizeof(P));
  const uintptr_t a = (uintptr_t)d_in;
  P.mis = (int32_t)((a & 15u) >> 2);
  P.abase = (const int32_t*)(a - (a & 15u));
  P.n = n;
  P.d_n = d_n;
  P.hdr = (uint32_t*)d_ws;
  P.ticket = (unsigned long long*)((char*)d_ws + 8);
  P.status = (uint64_t*)((char*)d_ws + SEL_HDR_BYTES);
  bool ne = false;
  for (int o = 0; o < M; ++o) {
    P.lo[o] = cp[o].lo;
    P.span[o] = (uint32_t)cp[o].hi - (uint32_t)cp[o].lo;
    P.n_ne[o] = cp[o].n_ne;
    for (int j = 0; j < RA_MAX_PREDS; ++j) P.ne[o][j] = j < cp[o].n_ne ? cp[o].ne[j] : 0;
    if (cp[o].lo > cp[o].hi) {  // empty interval: x == 0 and x != 0
      P.lo[o] = 0;
      P.span[o] = 0;
      P.n_ne[o] = 1;
      P.ne[o][0] = 0;
    }
    ne |= P.n_ne[o] > 0;
    P.out[o] = d_outs[o];
    P.out_cap[o] = out_caps[o];
    P.d_count[o] = d_counts[o];
  }
  const int64_t tile = mo_tile_rows(M);
  const int64_t ntiles = n > 0 ? (n + P.mis + tile - 1) / tile : 0;
  switch (M * 2 + (ne ? 1 : 0)) {
    case 2: return launch_mo<1, false>(P, ntiles, s);
    case 3: return launch_mo<1, true>(P, ntiles, s);
    case 4: return launch_mo<2, false>(P, ntiles, s);
    case 5: return launch_mo<2, true>(P, ntiles, s);
    case 6: return launch_mo<3, false>(P, ntiles, s);
    case 7: return launch_mo<3, true>(P, ntiles, s);
    case 8: return launch_mo<4, false>(P, ntiles, s);
    default: return launch_mo<4, true>(P, ntiles, s);
  }
}

}  // namespace ra

#ifdef RA_MO_PROFILE
// diagnostics build only: read and reset the counters (scripts/mo_prof.py)
extern "C" __attribute__((visibility("default"))) int ramo_prof(unsigned long long* out64) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out64, ra::g_mo_prof, sizeof(unsigned long long) * 32);
  cudaMemcpyFromSymbol(out64 + 32, ra::g_mo_cnt, sizeof(unsigned long long) * 32);
  unsigned long long z[32] = {};
  cudaMemcpyToSymbol(ra::g_mo_prof, z, sizeof(z));
  cudaMemcpyToSymbol(ra::g_mo_cnt, z, sizeof(z));
  return 0;
}
#endif
