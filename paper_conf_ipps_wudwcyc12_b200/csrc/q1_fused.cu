// q1_fused.cu — TPC-H Q1 as one fused kernel for sm_100a.
//
// The paper's Q1 plan (Fig 17(a), §V) is SELECT + six
// JOINs (fused) -> SORT by (returnflag, linestatus) -> fused arithmetic ->
// aggregate/unique; SORT alone was ~71% of the baseline (L1576-1577) and the
// fusible part gained 3.18x (L1673-1676).  In a positional column store the
// JOINs are identities and the SORT only orders <= 6 groups, so
// the whole query becomes one streaming pass:
//
//   SELECT   shipdate <= cutoff                              (Fig 2(g))
//   PROJECT  disc_price = price*(100-disc), charge = disc_price*(100+tax)
//            computed in registers, never stored             (Fig 2(h))
//   GROUP BY slot = 2*rf + ls into per-thread register accumulators (6 slots),
//            reduced warp -> CTA -> grid at the end; the last CTA to finish
//            folds the CTA partials (threadfence + ticket) in 128-bit.
//
// Two kernels compute exactly the same thing:
//
// * q1_tma_kernel (the hot path): persistent, one CTA per SM, warp-specialised.
//   A producer warp streams 1024-row tiles of all seven columns (38 B/row,
//   seven cp.async.bulk copies per tile) through a 4-stage shared-memory ring
//   completed on mbarriers, so ~117 KB per SM are always in flight and the
//   compute warps never wait on HBM latency; 8 compute warps read their rows
//   from shared memory and release the stage on an "empty" mbarrier.
//   Accumulators are narrowed: per row, count and discount share one 32-bit
//   add, quantity and price are 32-bit adds while both are "narrow"
//   (quantity < 2^16, price < 2^24 — every TPC-H row), flushed every 256 rows
//   into per-thread 64-bit sums in shared memory; wider (still in-domain)
//   values go straight to those 64-bit sums.  disc_price and charge stay
//   64-bit in registers.  ~8 instead of ~11 instructions per slot per row.
// * q1_grid_kernel: grid-stride over 4-row groups with 128-bit register
//   loads; used when the seven columns cannot all be 16-B aligned at a common
//   row (the bulk copies need that) or when the input is smaller than a tile.
//
// Exactness: in the documented domain (ra.h) a row's
// disc_price < 2^38 and charge < 2^46.  Each thread handles <= 2^17 rows
// (enforced by the grid size for n < 2^32) so its 64-bit sums cannot wrap;
// warp, CTA and grid sums of disc_price and charge are 128-bit.

#include <stdio.h>

#include "q1_common.cuh"

namespace ra {

namespace {

using namespace q1c;

struct Q1Params {
  const int32_t* sd;
  const uint8_t* rf;
  const uint8_t* ls;
  const int64_t* q;
  const int64_t* p;
  const int64_t* d;
  const int64_t* t;
  int64_t n;
  int64_t head;     // rows before the first aligned row (scalar path)
  int64_t ngroups;  // grid kernel: aligned 4-row groups; TMA kernel: full tiles
  int32_t cutoff;
  ra_q1_partial* out;
  int accumulate;  // add into *out (chunks of one query under fission) instead of overwriting
  unsigned long long* acc;  // grid accumulators [NS][ACC_K] (q1_common.cuh)
  uint32_t* counter;        // [0] CTA ticket, [1] status
};

// Per-row SELECT + domain checks + group slot + PROJECT.  Returns the slot
// (-1: not accumulated) and the projected disc_price / charge.
struct RowVal {
  int slot;
  uint64_t dp, ch;
};

__device__ __forceinline__ RowVal classify(uint32_t& status, int32_t cutoff, int32_t sd, uint32_t rfb, uint32_t lsb,
                                           int64_t q, int64_t p, int64_t d, int64_t t) {
  const bool sel = sd <= cutoff;  // SELECT
  // branch-free flag decode: rf A/N/R -> 0/2/4, ls F/O -> 0/1
  const uint32_t isN = rfb == 'N', isR = rfb == 'R';
  const bool okf = ((rfb == 'A') | isN | isR) & ((lsb == 'F') | (lsb == 'O'));
  const bool okn = ((uint64_t)q < (1ull << 31)) & ((uint64_t)p < (1ull << 31)) &
                   ((uint64_t)d <= 100ull) & ((uint64_t)t <= 100ull);
  status |= sel ? ((okf ? 0u : 1u) | (okn ? 0u : 2u)) : 0u;
  RowVal v;
  v.slot = (sel & okf & okn) ? (int)(2 * isN + 4 * isR + (lsb == 'O')) : -1;
  // PROJECT (exact in the domain: 32x32->64 and 64x32 products)
  v.dp = (uint64_t)(uint32_t)p * (uint32_t)(100 - (uint32_t)d);
  v.ch = v.dp * (uint64_t)(100u + (uint32_t)t);
  return v;
}

// Predicated slot update (one setp + predicated adds).  Written in PTX
// because nvcc otherwise lowers the 6-way one-hot update to an indirect
// jump table (BRX), i.e. a divergent branch per row.
template <int S>
__device__ __forceinline__ void padd_3x32_2x64(int slot, uint32_t& a, uint32_t& b, uint32_t& c, uint64_t& x,
                                               uint64_t& y, uint32_t va, uint32_t vb, uint32_t vc, uint64_t vx,
                                               uint64_t vy) {
  asm("{\n\t.reg .pred p;\n\t"
      "setp.eq.s32 p, %5, %6;\n\t"
      "@p add.u32 %0, %0, %7;\n\t"
      "@p add.u32 %1, %1, %8;\n\t"
      "@p add.u32 %2, %2, %9;\n\t"
      "@p add.u64 %3, %3, %10;\n\t"
      "@p add.u64 %4, %4, %11;\n\t}"
      : "+r"(a), "+r"(b), "+r"(c), "+l"(x), "+l"(y)
      : "r"(slot), "n"(S), "r"(va), "r"(vb), "r"(vc), "l"(vx), "l"(vy));
}

template <int S>
__device__ __forceinline__ void padd_2x32_4x64(int slot, uint32_t& a, uint32_t& b, uint64_t& w, uint64_t& x,
                                               uint64_t& y, uint64_t& z, uint32_t va, uint32_t vb, uint64_t vw,
                                               uint64_t vx, uint64_t vy, uint64_t vz) {
  asm("{\n\t.reg .pred p;\n\t"
      "setp.eq.s32 p, %6, %7;\n\t"
      "@p add.u32 %0, %0, %8;\n\t"
      "@p add.u32 %1, %1, %9;\n\t"
      "@p add.u64 %2, %2, %10;\n\t"
      "@p add.u64 %3, %3, %11;\n\t"
      "@p add.u64 %4, %4, %12;\n\t"
      "@p add.u64 %5, %5, %13;\n\t}"
      : "+r"(a), "+r"(b), "+l"(w), "+l"(x), "+l"(y), "+l"(z)
      : "r"(slot), "n"(S), "r"(va), "r"(vb), "l"(vw), "l"(vx), "l"(vy), "l"(vz));
}

__device__ __forceinline__ void row(Acc& A, int32_t cutoff, int32_t sd, uint32_t rfb, uint32_t lsb, int64_t q,
                                    int64_t p, int64_t d, int64_t t) {
  const RowVal v = classify(A.status, cutoff, sd, rfb, lsb, q, p, d, t);
  // GROUP BY into register slots (predicated adds)
#define Q1_SLOT(S)                                                                                          \
  padd_2x32_4x64<S>(v.slot, A.cnt[S], A.sdisc[S], A.sq[S], A.sp[S], A.sdp[S], A.sch[S], 1u, (uint32_t)d, \
                    (uint64_t)q, (uint64_t)p, v.dp, v.ch)
  Q1_SLOT(0); Q1_SLOT(1); Q1_SLOT(2); Q1_SLOT(3); Q1_SLOT(4); Q1_SLOT(5);
#undef Q1_SLOT
}

// ===================================================== grid-stride kernel
constexpr int Q1G_THREADS = 256;

struct Group4 {
  int4 sd;
  uint32_t rf, ls;
  longlong2 q[2], p[2], d[2], t[2];
};

__device__ __forceinline__ longlong2 ld_stream_ll2(const int64_t* ptr) {
  longlong2 r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.s64 {%0,%1}, [%2];" : "=l"(r.x), "=l"(r.y) : "l"(ptr));
  return r;
}

__device__ __forceinline__ uint32_t ld_stream_u32(const uint8_t* ptr) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(ptr));
  return r;
}

__device__ __forceinline__ void load_group(Group4& G, const Q1Params& P, int64_t g) {
  const int64_t r = P.head + 4 * g;
  G.sd = dev::ld_stream_v4((const int4*)(P.sd + r));
  G.rf = ld_stream_u32(P.rf + r);
  G.ls = ld_stream_u32(P.ls + r);
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    G.q[h] = ld_stream_ll2(P.q + r + 2 * h);
    G.p[h] = ld_stream_ll2(P.p + r + 2 * h);
    G.d[h] = ld_stream_ll2(P.d + r + 2 * h);
    G.t[h] = ld_stream_ll2(P.t + r + 2 * h);
  }
}

__device__ __forceinline__ void process_group(Acc& A, const Group4& G, int32_t cutoff) {
  row(A, cutoff, G.sd.x, G.rf & 0xFF, G.ls & 0xFF, G.q[0].x, G.p[0].x, G.d[0].x, G.t[0].x);
  row(A, cutoff, G.sd.y, (G.rf >> 8) & 0xFF, (G.ls >> 8) & 0xFF, G.q[0].y, G.p[0].y, G.d[0].y, G.t[0].y);
  row(A, cutoff, G.sd.z, (G.rf >> 16) & 0xFF, (G.ls >> 16) & 0xFF, G.q[1].x, G.p[1].x, G.d[1].x, G.t[1].x);
  row(A, cutoff, G.sd.w, G.rf >> 24, G.ls >> 24, G.q[1].y, G.p[1].y, G.d[1].y, G.t[1].y);
}

__global__ void __launch_bounds__(Q1G_THREADS, 2) q1_grid_kernel(const Q1Params P) {
  dev::grid_dep_wait();  // launch_pdl: the previous kernel's writes (e.g. a running partial) are visible
  __shared__ uint64_t s_w[Q1G_THREADS / 32][NS][8];
  __shared__ uint32_t s_status;
  __shared__ bool s_last;

  Acc A;
  acc_zero(A);
  const int64_t gtid = (int64_t)blockIdx.x * Q1G_THREADS + threadIdx.x;
  const int64_t gstride = (int64_t)gridDim.x * Q1G_THREADS;

  // aligned 4-row groups (10 x 128-bit loads in flight per thread per group)
  for (int64_t g = gtid; g < P.ngroups; g += gstride) {
    Group4 G0;
    load_group(G0, P, g);
    process_group(A, G0, P.cutoff);
  }
  // scalar rows: [0, head) and the tail after the aligned groups
  const int64_t tail0 = P.head + 4 * P.ngroups;
  const int64_t nscalar = P.head + (P.n - tail0);
  for (int64_t i = gtid; i < nscalar; i += gstride) {
    const int64_t r = i < P.head ? i : tail0 + (i - P.head);
    row(A, P.cutoff, P.sd[r], P.rf[r], P.ls[r], P.q[r], P.p[r], P.d[r], P.t[r]);
  }
  reduce_and_fold<Q1G_THREADS / 32>(A, P, s_w, &s_status, &s_last);
}

// ============================================================ TMA kernel
constexpr int Q1T_NT = 256;        // compute threads (8 warps) + 1 producer warp
constexpr int Q1T_TILE = 1024;     // rows per tile (38 KB of columns)
constexpr int Q1T_STAGES = 4;      // shared-memory ring depth
constexpr int Q1T_FLUSH = 256;     // rows per thread between narrow -> wide flushes
constexpr int Q1T_NW = Q1T_NT / 32;
constexpr int Q1T_R = Q1T_TILE / Q1T_NT;  // rows per thread per tile (pairs of 2)
static_assert(Q1T_R % 2 == 0, "rows per thread per tile must be even");
constexpr int Q1T_FLUSH_TILES = Q1T_FLUSH / Q1T_R;

// stage layout (bytes): q, p, d, t int64[T] | shipdate int32[T] | rf u8[T] | ls u8[T]
constexpr int OFF_Q = 0, OFF_P = 8 * Q1T_TILE, OFF_D = 16 * Q1T_TILE, OFF_T = 24 * Q1T_TILE;
constexpr int OFF_SD = 32 * Q1T_TILE, OFF_RF = 36 * Q1T_TILE, OFF_LS = 37 * Q1T_TILE;
constexpr int STAGE_BYTES = 38 * Q1T_TILE;

struct Q1TmaSmem {
  alignas(128) unsigned char stage[Q1T_STAGES][STAGE_BYTES];
  // per-thread 64-bit sums: (cnt<<32 | disc), qty, price, disc_price, charge
  uint64_t wide[5][NS][Q1T_NT];
  uint64_t s_w[Q1T_NW][NS][8];
  uint64_t full[Q1T_STAGES], empty[Q1T_STAGES];
  uint32_t status;
  bool last;
};
constexpr size_t Q1T_SMEM = sizeof(Q1TmaSmem);
static_assert(Q1T_SMEM <= 227 * 1024, "Q1 TMA kernel exceeds the shared-memory opt-in limit");

// Fast-path per-thread accumulators (see the header comment).  Between two
// flushes a thread adds <= Q1T_FLUSH = 256 rows; with disc_price dp < 2^31
// split as dp = dh * 2^16 + dl (dh < 2^15, dl < 2^16) and f = 100 + tax
// <= 200, every sum below stays within 32 bits:
struct NarrowAcc {
  uint32_t cd[NS];   // count << 16 | discount sum  (count <= 256, disc sum <= 25600)
  uint32_t q[NS];    // quantity                    (< 2^16 * 2^8)
  uint32_t p[NS];    // price                       (<= (2^24 - 1) * 2^8 < 2^32)
  uint32_t dh[NS];   // disc_price >> 16            (< 2^15 * 2^8)
  uint32_t dl[NS];   // disc_price & 0xffff         (< 2^16 * 2^8)
  uint32_t chh[NS];  // f * (dp >> 16)              (< 200 * 2^15 * 2^8 < 2^31)
  uint32_t chl[NS];  // f * (dp & 0xffff)           (< 200 * 2^16 * 2^8 < 2^32)
  uint64_t dp[NS];   // flushed disc_price          (< 2^31 * 2^17 rows/thread)
  uint64_t ch[NS];   // flushed charge              (< 2^39 * 2^17)
};

// One predicated slot update: seven 32-bit adds under one predicate.  PTX
// because nvcc otherwise turns the 6-way one-hot update into an indirect
// jump table (BRX), i.e. a divergent branch per row.
template <int S>
__device__ __forceinline__ void fast_slot(NarrowAcc& A, int slot, uint32_t cdv, uint32_t q, uint32_t p, uint32_t dh,
                                          uint32_t dl, uint32_t chh, uint32_t chl) {
  asm("{\n\t.reg .pred p;\n\t"
      "setp.eq.s32 p, %7, %8;\n\t"
      "@p add.u32 %0, %0, %9;\n\t"
      "@p add.u32 %1, %1, %10;\n\t"
      "@p add.u32 %2, %2, %11;\n\t"
      "@p add.u32 %3, %3, %12;\n\t"
      "@p add.u32 %4, %4, %13;\n\t"
      "@p add.u32 %5, %5, %14;\n\t"
      "@p add.u32 %6, %6, %15;\n\t}"
      : "+r"(A.cd[S]), "+r"(A.q[S]), "+r"(A.p[S]), "+r"(A.dh[S]), "+r"(A.dl[S]), "+r"(A.chh[S]), "+r"(A.chl[S])
      : "r"(slot), "n"(S), "r"(cdv), "r"(q), "r"(p), "r"(dh), "r"(dl), "r"(chh), "r"(chl));
}

// Fast path of one row: accumulates it iff it is selected, its flags are in
// {A,N,R} x {F,O}, and its numbers are narrow (0 <= quantity < 2^16,
// 0 <= price < 2^24, 0 <= discount, tax <= 100 — every TPC-H row).
// Returns true for a selected row it did NOT take (the caller's slow path
// then classifies it exactly: domain status bits or 64-bit sums).
__device__ __forceinline__ bool fast_row(NarrowAcc& A, int32_t cutoff, int32_t sd, uint32_t rfb, uint32_t lsb,
                                         int64_t q, int64_t p, int64_t d, int64_t t) {
  const uint32_t ql = (uint32_t)q, pl = (uint32_t)p, dl = (uint32_t)d, tl = (uint32_t)t;
  const uint32_t hi = (uint32_t)((uint64_t)q >> 32) | (uint32_t)((uint64_t)p >> 32) |
                      (uint32_t)((uint64_t)d >> 32) | (uint32_t)((uint64_t)t >> 32);
  const bool sel = sd <= cutoff;  // SELECT
  const bool num = ((ql | (pl >> 8) | hi) < (1u << 16)) & (dl <= 100u) & (tl <= 100u);
  const bool isN = rfb == 'N', isR = rfb == 'R', isO = lsb == 'O';
  const bool flags = (isN | isR | (rfb == 'A')) & (isO | (lsb == 'F'));
  const bool fast = sel & num & flags;
  const int slot = fast ? (isN ? 2 : 0) + (isR ? 4 : 0) + (isO ? 1 : 0) : -1;
  // PROJECT: disc_price = price * (100 - disc) < 2^31, charge = disc_price * f
  const uint32_t dp = pl * (100u - dl), f = 100u + tl;
  const uint32_t dph = dp >> 16, dpl = dp & 0xFFFFu;
  const uint32_t cdv = (1u << 16) | dl;
  const uint32_t chh = f * dph, chl = f * dpl;
  fast_slot<0>(A, slot, cdv, ql, pl, dph, dpl, chh, chl);
  fast_slot<1>(A, slot, cdv, ql, pl, dph, dpl, chh, chl);
  fast_slot<2>(A, slot, cdv, ql, pl, dph, dpl, chh, chl);
  fast_slot<3>(A, slot, cdv, ql, pl, dph, dpl, chh, chl);
  fast_slot<4>(A, slot, cdv, ql, pl, dph, dpl, chh, chl);
  fast_slot<5>(A, slot, cdv, ql, pl, dph, dpl, chh, chl);
  return sel & !fast;
}

// Slow path of one selected row the fast path did not take: the exact domain
// classification (status bits, ra.h) and, when in the domain, 64-bit adds
// into the thread's private sums in shared memory.
__device__ __forceinline__ void slow_row(Q1TmaSmem& S, uint32_t& status, int tid, int32_t cutoff, int32_t sd,
                                         uint32_t rfb, uint32_t lsb, int64_t q, int64_t p, int64_t d, int64_t t) {
  const RowVal v = classify(status, cutoff, sd, rfb, lsb, q, p, d, t);
  if (v.slot < 0) return;
  S.wide[0][v.slot][tid] += (1ull << 32) | (uint64_t)d;
  S.wide[1][v.slot][tid] += (uint64_t)q;
  S.wide[2][v.slot][tid] += (uint64_t)p;
  S.wide[3][v.slot][tid] += v.dp;
  S.wide[4][v.slot][tid] += v.ch;
}

__device__ __forceinline__ void flush(NarrowAcc& A, Q1TmaSmem& S, int tid) {
#pragma unroll
  for (int s = 0; s < NS; ++s) {
    S.wide[0][s][tid] += ((uint64_t)(A.cd[s] >> 16) << 32) | (A.cd[s] & 0xFFFFu);
    S.wide[1][s][tid] += A.q[s];
    S.wide[2][s][tid] += A.p[s];
    A.dp[s] += ((uint64_t)A.dh[s] << 16) + A.dl[s];
    A.ch[s] += ((uint64_t)A.chh[s] << 16) + A.chl[s];
    A.cd[s] = A.q[s] = A.p[s] = A.dh[s] = A.dl[s] = A.chh[s] = A.chl[s] = 0;
  }
}

__global__ void __launch_bounds__(Q1T_NT + 32, 1) q1_tma_kernel(const Q1Params P) {
  dev::grid_dep_wait();  // launch_pdl: the previous kernel's writes (e.g. a running partial) are visible
  extern __shared__ __align__(128) unsigned char q1_smem_raw[];
  Q1TmaSmem& S = *reinterpret_cast<Q1TmaSmem*>(q1_smem_raw);
  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31;
  const int64_t ntiles = P.ngroups;

  if (tid == 0) {
    for (int s = 0; s < Q1T_STAGES; ++s) {
      dev::mbar_init(&S.full[s], 1);
      dev::mbar_init(&S.empty[s], Q1T_NW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (tid < Q1T_NT) {
#pragma unroll
    for (int f = 0; f < 5; ++f)
#pragma unroll
      for (int s = 0; s < NS; ++s) S.wide[f][s][tid] = 0;
  }
  __syncthreads();

  Acc A;
  acc_zero(A);
  if (warp == Q1T_NW) {
    // ---------------- producer warp: one elected lane issues the bulk copies
    if (lane == 0) {
      int i = 0;
      for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
        const int s = i % Q1T_STAGES;
        if (i >= Q1T_STAGES) dev::mbar_wait(&S.empty[s], ((i / Q1T_STAGES) + 1) & 1);
        const int64_t r0 = P.head + tile * Q1T_TILE;
        unsigned char* st = S.stage[s];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        dev::mbar_arrive_expect_tx(&S.full[s], STAGE_BYTES);
        dev::bulk_g2s(st + OFF_Q, P.q + r0, 8 * Q1T_TILE, &S.full[s]);
        dev::bulk_g2s(st + OFF_P, P.p + r0, 8 * Q1T_TILE, &S.full[s]);
        dev::bulk_g2s(st + OFF_D, P.d + r0, 8 * Q1T_TILE, &S.full[s]);
        dev::bulk_g2s(st + OFF_T, P.t + r0, 8 * Q1T_TILE, &S.full[s]);
        dev::bulk_g2s(st + OFF_SD, P.sd + r0, 4 * Q1T_TILE, &S.full[s]);
        dev::bulk_g2s(st + OFF_RF, P.rf + r0, Q1T_TILE, &S.full[s]);
        dev::bulk_g2s(st + OFF_LS, P.ls + r0, Q1T_TILE, &S.full[s]);
      }
    }
  } else {
    // ---------------- compute warps
    NarrowAcc N;
#pragma unroll
    for (int s = 0; s < NS; ++s) {
      N.cd[s] = N.q[s] = N.p[s] = N.dh[s] = N.dl[s] = N.chh[s] = N.chl[s] = 0;
      N.dp[s] = N.ch[s] = 0;
    }
    uint32_t status = 0;
    int i = 0, since = 0;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
      const int s = i % Q1T_STAGES;
      dev::mbar_wait(&S.full[s], (i / Q1T_STAGES) & 1);
      const unsigned char* st = S.stage[s];
#pragma unroll
      for (int m = 0; m < Q1T_R / 2; ++m) {
        const int r = 2 * (tid + m * Q1T_NT);  // rows r, r+1 of the tile
        const int2 sd = *reinterpret_cast<const int2*>(st + OFF_SD + 4 * r);
        const uint32_t rf = *reinterpret_cast<const uint16_t*>(st + OFF_RF + r);
        const uint32_t ls = *reinterpret_cast<const uint16_t*>(st + OFF_LS + r);
        const longlong2 q = *reinterpret_cast<const longlong2*>(st + OFF_Q + 8 * r);
        const longlong2 p = *reinterpret_cast<const longlong2*>(st + OFF_P + 8 * r);
        const longlong2 d = *reinterpret_cast<const longlong2*>(st + OFF_D + 8 * r);
        const longlong2 t = *reinterpret_cast<const longlong2*>(st + OFF_T + 8 * r);
        const bool w0 = fast_row(N, P.cutoff, sd.x, rf & 0xFF, ls & 0xFF, q.x, p.x, d.x, t.x);
        const bool w1 = fast_row(N, P.cutoff, sd.y, rf >> 8, ls >> 8, q.y, p.y, d.y, t.y);
        if (__any_sync(0xffffffffu, w0 | w1)) {  // warp-uniform, rare (never for TPC-H data)
          if (w0) slow_row(S, status, tid, P.cutoff, sd.x, rf & 0xFF, ls & 0xFF, q.x, p.x, d.x, t.x);
          if (w1) slow_row(S, status, tid, P.cutoff, sd.y, rf >> 8, ls >> 8, q.y, p.y, d.y, t.y);
        }
      }
      __syncwarp();
      if (lane == 0) dev::mbar_arrive(&S.empty[s]);
      if (++since == Q1T_FLUSH_TILES) {
        flush(N, S, tid);
        since = 0;
      }
    }
    flush(N, S, tid);
    // scalar rows: [0, head) and the tail after the full tiles (< 1 per thread)
    const int64_t tail0 = P.head + ntiles * Q1T_TILE;
    const int64_t nscalar = P.head + (P.n - tail0);
    for (int64_t j = (int64_t)blockIdx.x * Q1T_NT + tid; j < nscalar; j += (int64_t)gridDim.x * Q1T_NT) {
      const int64_t r = j < P.head ? j : tail0 + (j - P.head);
      const int32_t sd = P.sd[r];
      const uint32_t rfb = P.rf[r], lsb = P.ls[r];
      const int64_t q = P.q[r], p = P.p[r], d = P.d[r], t = P.t[r];
      if (fast_row(N, P.cutoff, sd, rfb, lsb, q, p, d, t)) slow_row(S, status, tid, P.cutoff, sd, rfb, lsb, q, p, d, t);
    }
    flush(N, S, tid);
#pragma unroll
    for (int s = 0; s < NS; ++s) {
      const uint64_t w0 = S.wide[0][s][tid];
      A.cnt[s] = (uint32_t)(w0 >> 32);
      A.sdisc[s] = (uint32_t)w0;
      A.sq[s] = S.wide[1][s][tid];
      A.sp[s] = S.wide[2][s][tid];
      A.sdp[s] = N.dp[s] + S.wide[3][s][tid];
      A.sch[s] = N.ch[s] + S.wide[4][s][tid];
    }
    A.status = status;
  }
  reduce_and_fold<Q1T_NW>(A, P, S.s_w, &S.status, &S.last);
}

std::atomic<int> g_q1_occ[64];   // blocks/SM of the grid kernel per device (0 = unknown)
std::atomic<int> g_q1_attr[64];  // 1: dynamic smem opt-in done for the TMA kernel

// First row h < 16 at which every column is 16-B aligned (flags included),
// or -1.  `flag_align` = required alignment of the flag columns.
int64_t common_head(const ra_lineitem& c, int64_t n, int flag_align) {
  for (int64_t h = 0; h < 16 && h < n; ++h) {
    const bool ok = ((uintptr_t)(c.shipdate + h) % 16 == 0) &&
                    ((uintptr_t)(c.returnflag + h) % flag_align == 0) &&
                    ((uintptr_t)(c.linestatus + h) % flag_align == 0) && ((uintptr_t)(c.quantity + h) % 16 == 0) &&
                    ((uintptr_t)(c.extendedprice + h) % 16 == 0) && ((uintptr_t)(c.discount + h) % 16 == 0) &&
                    ((uintptr_t)(c.tax + h) % 16 == 0);
    if (ok) return h;
  }
  return -1;
}

}  // namespace

size_t q1_ws_bytes() { return 256 + (size_t)Q1_MAX_GRID * sizeof(Q1Block); }
size_t q1_ws_clear_bytes() { return ACC_OFFSET + sizeof(unsigned long long) * NS * ACC_K; }
static_assert(ACC_OFFSET + sizeof(unsigned long long) * NS * ACC_K <= 256 + Q1_MAX_GRID * sizeof(Q1Block),
              "accumulators inside the Q1 workspace");

int launch_q1(const ra_lineitem& c, int64_t n, int32_t cutoff, ra_q1_partial* d_partial, void* d_ws,
              size_t ws_bytes, cudaStream_t s, int accumulate) {
  (void)ws_bytes;
  Q1Params P;
  P.sd = c.shipdate;
  P.rf = c.returnflag;
  P.ls = c.linestatus;
  P.q = c.quantity;
  P.p = c.extendedprice;
  P.d = c.discount;
  P.t = c.tax;
  P.n = n;
  P.cutoff = cutoff;
  P.out = d_partial;
  P.accumulate = accumulate;
  P.counter = (uint32_t*)d_ws;
  P.acc = (unsigned long long*)((char*)d_ws + ACC_OFFSET);
  const int dev = current_device();
  // per-thread 64-bit sums stay exact while rows/thread <= 2^17
  const int64_t sms = num_sms();

  // ---- TMA kernel: needs one row at which all seven columns are 16-B aligned
  const int64_t h16 = common_head(c, n, 16);
  if (h16 >= 0 && (n - h16) / Q1T_TILE >= 1) {
    P.head = h16;
    P.ngroups = (n - h16) / Q1T_TILE;
    const int a = device_once(g_q1_attr, dev, [] {
      cudaError_t e = cudaFuncSetAttribute(q1_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Q1T_SMEM);
      return e != cudaSuccess ? cuda_fail(e, "q1_tma_kernel smem attribute") : 1;
    });
    if (a < 0) return a;
    int64_t grid = sms < P.ngroups ? sms : P.ngroups;
    const int64_t min_grid = (n >> 17) / Q1T_NT + 1;
    if (grid < min_grid) grid = min_grid;
    if (grid > Q1_MAX_GRID) return fail(RA_E_INVAL, "n too large for the Q1 grid");
    cudaError_t e = launch_pdl(q1_tma_kernel, dim3((unsigned)grid), dim3(Q1T_NT + 32), Q1T_SMEM, s, P);
    count_launch();
    if (e != cudaSuccess) return cuda_fail(e, "q1_tma_kernel launch");
    return RA_OK;
  }

  // ---- grid-stride kernel (columns not co-alignable, or fewer rows than a tile)
  const int64_t h4 = common_head(c, n, 4);
  P.head = h4 >= 0 ? h4 : n;
  P.ngroups = h4 >= 0 ? (n - h4) / 4 : 0;
  const int occ = device_once(g_q1_occ, dev, [] {
    int o = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, q1_grid_kernel, Q1G_THREADS, 0);
    return e != cudaSuccess ? cuda_fail(e, "occupancy query") : (o > 0 ? o : 1);
  });
  if (occ < 0) return occ;
  int64_t grid = sms * occ;
  if (grid > Q1_MAX_GRID) grid = Q1_MAX_GRID;
  const int64_t work = P.ngroups > 0 ? P.ngroups : n;
  const int64_t need = (work + Q1G_THREADS - 1) / Q1G_THREADS;
  if (grid > need) grid = need;
  const int64_t min_grid = (n >> 17) / Q1G_THREADS + 1;
  if (grid < min_grid) grid = min_grid;
  if (grid < 1) grid = 1;
  if (grid > Q1_MAX_GRID) return fail(RA_E_INVAL, "n too large for the Q1 grid");
  cudaError_t e = launch_pdl(q1_grid_kernel, dim3((unsigned)grid), dim3(Q1G_THREADS), 0, s, P);
  count_launch();
  if (e != cudaSuccess) return cuda_fail(e, "q1_grid_kernel launch");
  return RA_OK;
}

}  // namespace ra
