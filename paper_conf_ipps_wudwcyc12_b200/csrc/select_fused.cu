// select_fused.cu — single-pass, single-output SELECT for sm_100a: the
// tuple SELECT's key pass (row ids + order masks for the payload compaction)
// and every SELECT pass over at most 2^21 rows (fused chain or one pass of the
// unfused chain), where its lighter launch wins.  Larger fused chains, the
// unfused chain's larger passes and several SELECTs on one input run
// select_multi.cu's warp-specialised pass (writer warps, cooperative
// look-back), measured faster on B200.
//
// The paper's SELECT has four stages — partition, filter, buffer, gather —
// in two CUDA kernels separated by a global synchronisation so that each CTA
// can find "the correct position in the final array" of its matches
// (Fig 3).  Fusing a chain inserts further filter
// stages after the first and keeps one partition/buffer/gather
// (Fig 6; L784-785, L812-814).
//
// Here the whole chain is ONE persistent, warp-specialised kernel: two CTAs per
// SM, each with 8 compute warps, one producer warp and one look-back warp.
//
//   partition  the producer warp draws 8192-row tiles from an atomic ticket
//              counter (one ticket ahead, so the atomic's round trip overlaps
//              the wait for a free slot); a CTA that runs slow simply takes
//              fewer tiles: no tile ever waits on a CTA that is far behind.
//   load       each tile arrives by one 1-D bulk async copy (cp.async.bulk, TMA
//              engine) into a 2-slot shared-memory ring completed on mbarriers;
//              a slot is refilled as soon as the compute warps have read it, so
//              up to two 32 KB tiles per CTA (128 KB per SM) are in flight.
//   filter     each compute warp owns 1024 contiguous rows of the tile, read as
//              eight conflict-free 128-bit shared loads per lane; the folded
//              predicate (lo <= x <= hi, x != ne[]) is evaluated in registers.
//   buffer     packed 5-step warp scans (4 rows x 8 bits per word) and a
//              warp-count reduction order the matches; they are compacted into a
//              40 KB shared-memory ring of selected rows (variable size per
//              tile, each run contiguous) and the tile aggregate is published at
//              once.
//   gather     once the look-back warp has placed a tile (its global offset),
//              the compute warps copy its run from the ring to the output with
//              coalesced stores.
//
// Look-back, B200 style.  An L2 round trip under full HBM load (~1.4 us) is
// comparable to a tile's time budget, so nothing on the compute path waits for
// one:
//   * exclusive(t) = inclusive(t') + the aggregates of the tiles strictly
//     between t' and t, where t' is this CTA's previous tile — whose inclusive
//     prefix the look-back warp holds in a register.  Only aggregates are read,
//     each published in its owner's count phase — never the result of another
//     CTA's look-back: there is no chain of dependent look-backs.  Tickets are
//     drawn in order, so every tile between t' and t was drawn before t and is
//     counted within a tile time or two of being drawn.
//   * the look-back warp bulk-copies tile k's window (~296 words on average,
//     up to 768 fit a slot) into shared memory once tile k+1 is counted — by
//     then nearly every word in it is published — and resolves it as soon as
//     the copy lands (or at once, on demand, when the compute warps already
//     wait for tile k); a word still unpublished is re-polled individually.
//   * compute warps write tile k when tile k+3 is counted, or earlier when the
//     ring of selected rows runs short (high selectivity).
// (Measured on B200, 2^28 rows, k=2, s=.25 overall: window slots of 320 words
// left ~30% of windows uncopied -> one dependent L2 round trip each, 0.257 ms;
// 768-word slots copied one tile late: 0.230 ms.  1 CTA/SM with deeper input
// rings is far slower (0.34 ms) — scripts/sel_variants.sh + scripts/gpu_selvar.sh.)
//
// Status words carry a 28-bit launch epoch (header word advanced by the last
// CTA to finish, so every CTA of a launch reads the same value), so stale words of earlier launches read as "not ready": no per-call
// memset and no second kernel.  The ticket counter is reset by the last CTA to
// finish.  The launch before the tag wraps to 0 clears every status word the
// workspace has held (header high-water mark), so tags never alias.

#include <stdio.h>
#include <stdlib.h>

#include <type_traits>

#include "ra_internal.cuh"

namespace ra {

#ifdef RA_SEL_PROFILE  // counters for scripts/micro/sel_prof.cu; never in the product build
__device__ unsigned long long g_sel_prof[16];
#define PROF_ADD(k, v) atomicAdd(&g_sel_prof[k], (unsigned long long)(v))
#define PT_BEGIN(var) const long long var = clock64()
#define PT_END(k, var, cond) \
  if (cond) PROF_ADD(k, clock64() - var)
#else
#define PROF_ADD(k, v)
#define PT_BEGIN(var)
#define PT_END(k, var, cond)
#endif

namespace {

// status word: [63:62] flag | [61:34] epoch tag | [33:0] aggregate
constexpr uint64_t FLAG_A = 1ull << 62;  // tile aggregate published
constexpr int TAG_SHIFT = 34;
constexpr uint64_t TAG_MASK = (1ull << 28) - 1;

// header: u32 epoch at word 0, u64 ticket counter at byte 8, u32 done counter at
// byte 16, u64 status-word high-water mark at byte 24
constexpr int H_EPOCH = 0;
constexpr int H_DONE = 4;
constexpr int H_HWM = 6;

constexpr int NW = SEL_THREADS / 32;     // compute warps
constexpr int WROWS = SEL_TILE / NW;     // contiguous rows owned by a compute warp (1024)
constexpr int LBWARP = NW;               // look-back warp
constexpr int PRWARP = NW + 1;           // producer warp: tickets + bulk copies
constexpr int BLOCK = SEL_THREADS + 64;  // + the look-back and producer warps
#ifndef RA_SEL_LAG
#define RA_SEL_LAG 3
#endif
constexpr int LAG = RA_SEL_LAG;          // tile k is written when tile k+LAG is counted (or earlier)
constexpr int K = LAG + 2;               // metadata slots: tiles counted but not yet written
#ifndef RA_SEL_SMALL_ROWS_DEFAULT
#define RA_SEL_SMALL_ROWS_DEFAULT (1ll << 21)  // fused chains up to this many rows run select_fused_kernel
#endif
#ifndef RA_SEL_PDL
#define RA_SEL_PDL 1
#endif
#ifndef RA_SEL_PTXSCATTER
#define RA_SEL_PTXSCATTER 1
#endif
#ifndef RA_SEL_BATCH
#define RA_SEL_BATCH 1  // tiles per ticket (see the producer warp)
#endif
#ifndef RA_SEL_D1
#define RA_SEL_D1 1
#define RA_SEL_D2 1
#endif
constexpr int D1 = RA_SEL_D1;            // window of tile k copied when tile k+D1 is counted
constexpr int D2 = RA_SEL_D2;            // ... and resolved when tile k+D2 is counted
#ifndef RA_SEL_Q
#define RA_SEL_Q (RA_SEL_D2 - RA_SEL_D1 + 1)
#endif
constexpr int Q = RA_SEL_Q;              // window slots (windows in flight)
constexpr int LBW = 10;                  // window words per lane per pass
#ifndef RA_SEL_WIN
#define RA_SEL_WIN 768
#endif
constexpr int WIN_WORDS = RA_SEL_WIN;     // window slot capacity (status words)
constexpr int PASS_WORDS = 32 * LBW;      // words summed per warp pass
static_assert(WIN_WORDS % 2 == 0, "16-B granules");
constexpr int NPK = SEL_VEC / 4;         // packed count words per lane (4 bytes: one per vector j)
static_assert(SEL_VEC == 8 || SEL_VEC == 4, "fl holds 4 bits per vector in 32 bits; counts in NPK words");
// vector j's 8-bit count: word NPK*o + q_of(j), byte b_of(j) (see the packing below)
__host__ __device__ constexpr int q_of(int j) { return NPK == 2 ? (j & 1) : 0; }
__host__ __device__ constexpr int b_of(int j) { return NPK == 2 ? (j >> 1) : ((j >> 1) | ((j & 1) << 1)); }
static_assert(NW <= 32, "one warp reduces the per-warp counts");
static_assert(LAG >= D2 + 1, "a tile is placed before it is due");
static_assert(SEL_OUTRING >= SEL_TILE, "a whole tile must fit the ring");

struct SelParams {
  const int32_t* abase;  // 16-B aligned base, = d_in - mis
  int64_t n;             // host bound on rows
  const int64_t* d_n;    // optional device row count (unfused passes)
  int32_t* out;
  int64_t out_cap;
  int64_t* d_count;
  uint32_t* hdr;
  unsigned long long* ticket;
  uint64_t* status;  // status[tile]
  int32_t mis;       // rows of d_in's 16-B chunk before d_in (0..3)
  uint32_t* rowids;  // ROWS mode (ra_select_rows): the ring holds row ids, written here (or NULL)
  // ROWS mode, payload compaction (compact.cu): per tile the lanes' flag words
  // fmask[t][256] and meta[t][12] = the warps' exclusive bases + the tile offset
  uint32_t* fmask;
  uint32_t* meta;
  int32_t lo;
  uint32_t span;  // hi - lo (the interval is never empty: see launch_select_pass)
  int32_t n_ne;
  int32_t ne[RA_MAX_PREDS];
};

template <int RING>
struct __align__(128) SelSmemT {
  static constexpr int kRing = RING;
  int4 in[SEL_INSLOTS][SEL_TILE / 4];  // input tiles (bulk-copy destination)
  int32_t ring[RING];                  // selected rows of counted, not yet written tiles
  uint64_t win[Q][WIN_WORDS];          // look-back windows (bulk-copied status words)
  uint64_t full[SEL_INSLOTS];          // TMA -> compute: tile landed (or end marker)
  uint64_t empty[SEL_INSLOTS];         // compute -> producer: slot read
  uint64_t winfull[Q];                 // TMA -> look-back: window landed
  uint64_t counted[K];                 // compute -> look-back: aggregate in cnt[], index in tidx[]
  uint64_t placed[K];                  // look-back -> compute: offset in goff[]
  int64_t tile_of[SEL_INSLOTS];        // ticket held by each input slot
  int64_t tidx[K];                     // tile index of CTA-local tile k (-1: no more tiles)
  int64_t wlo[Q], whi[Q];              // window bounds [lo, hi) of each window slot
  int64_t goff[K];                     // tile output offsets
  uint32_t wtot[2][NW];                // [tile parity][warp] selected counts
  int32_t cnt[K];                      // tile aggregates
  int32_t start[K];                    // tile run start in the ring
  int32_t rin[K];                      // ring rows of each tile (0 once past out_cap)
  uint32_t past[2];                    // [tile parity] ROWS: the tile's ids land past out_cap
  int64_t n;
  uint32_t epoch;
  int32_t demand;  // oldest tile the compute warps are waiting to write (-1: none yet)
  int32_t sat;     // ROWS: a resolved tile of this CTA ended at or past out_cap (monotone hint)
};
// A 40 KB ring (2 CTAs/SM).
using SelSmem = SelSmemT<SEL_OUTRING>;

using dev::smem_u32;
using dev::mbar_init;
using dev::mbar_arrive;
using dev::mbar_arrive_expect_tx;
using dev::mbar_wait;
using dev::mbar_test;
using dev::bulk_g2s;

__device__ __forceinline__ void st_relaxed_shared(int32_t* p, int32_t v) {
  asm volatile("st.relaxed.cta.shared.b32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}

__device__ __forceinline__ int32_t ld_relaxed_shared(const int32_t* p) {
  int32_t v;
  asm volatile("ld.relaxed.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}

// Compute warps synchronise among themselves only (named barrier 1).
__device__ __forceinline__ void compute_bar() { asm volatile("bar.sync 1, %0;" ::"n"(SEL_THREADS) : "memory"); }

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <bool HAS_NE>
__device__ __forceinline__ bool keep(int32_t x, const SelParams& P) {
  bool k = (uint32_t)x - (uint32_t)P.lo <= P.span;  // lo <= x <= hi (mod-2^32 difference)
  if (HAS_NE) {
#pragma unroll
    for (int j = 0; j < RA_MAX_PREDS; ++j)
      if (j < P.n_ne) k &= (x != P.ne[j]);
  }
  return k;
}

__device__ __forceinline__ int32_t comp(const int4& v, int c) {
  return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w;
}

// Store v at shared byte address a and advance a, iff (fl & mask) != 0.
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

// Issue the bulk copy of tile t into input slot s (one thread).
template <typename SM>
__device__ __forceinline__ void issue_tile(SM& S, const SelParams& P, int64_t nv, int64_t t, int s) {
  const int64_t v0 = t * SEL_TILE;
  int64_t rows = nv - v0;
  if (rows > SEL_TILE) rows = SEL_TILE;
  const uint32_t bytes = (uint32_t)((rows * 4 + 15) & ~15ll);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // the slot was last read by generic loads
  mbar_arrive_expect_tx(&S.full[s], bytes);
  bulk_g2s(&S.in[s][0], P.abase + v0, bytes, &S.full[s]);
}

// Look-back warp, lane 0: bulk-copy window [lo, hi) of status words into slot
// q (16-B aligned start: one extra word may precede lo).  A window longer than
// the slot (a CTA that ran slow) is not copied; it is read directly instead.
template <typename SM>
__device__ __forceinline__ void issue_window(SM& S, const SelParams& P, int64_t lo, int64_t hi, int q) {
  S.wlo[q] = lo;
  S.whi[q] = hi;
  const int64_t s0 = lo & ~1ll;
  PROF_ADD(14, hi - s0 > WIN_WORDS ? 1 : 0);
  PROF_ADD(15, hi > lo ? hi - lo : 0);
  if (hi <= lo || hi - s0 > WIN_WORDS) {
    mbar_arrive(&S.winfull[q]);
    return;
  }
  const uint32_t bytes = (uint32_t)(((hi - s0) * 8 + 15) & ~15ll);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_arrive_expect_tx(&S.winfull[q], bytes);
  bulk_g2s(&S.win[q][0], P.status + s0, bytes, &S.winfull[q]);
}

// Sum of the aggregates of tiles [lo, hi) (one warp).  An aggregate is
// <= SEL_TILE < 2^32, so a word published by this launch has its high half
// exactly `want` = (FLAG_A | tag) >> 32: readiness is one compare and each
// pass sums in 32 bits (one REDUX).  Words still unpublished are re-polled.
template <typename SM>
__device__ __forceinline__ int64_t window_sum(const SM& S, const SelParams& P, int q, int lane, uint32_t want) {
  const int64_t lo = S.wlo[q], hi = S.whi[q];
  const int64_t s0 = lo & ~1ll;
  const bool copied = hi > lo && hi - s0 <= WIN_WORDS;
  const uint64_t pad = (uint64_t)want << 32;  // a ready word with a zero aggregate
  int64_t total = 0;
  // lane l takes words base + l + 32c: conflict-free shared loads, and on the
  // copied path no branches (clamped addresses + selects)
  for (int64_t base = lo; base < hi; base += PASS_WORDS) {
    uint64_t w[LBW];
    if (copied) {
#pragma unroll
      for (int c = 0; c < LBW; ++c) {
        const int64_t idx = base + lane + 32 * c;
        const bool in = idx < hi;
        const uint64_t x = S.win[q][(in ? idx : lo) - s0];
        w[c] = in ? x : pad;
      }
    } else {
#pragma unroll
      for (int c = 0; c < LBW; ++c) {
        const int64_t idx = base + lane + 32 * c;
        w[c] = idx < hi ? dev::ld_relaxed_u64(P.status + idx) : pad;
      }
    }
    for (int spins = 0;; ++spins) {
      bool missing = false;
#pragma unroll
      for (int c = 0; c < LBW; ++c) missing |= (uint32_t)(w[c] >> 32) != want;
      if (!__any_sync(0xffffffffu, missing)) break;
      if (lane == 0) PROF_ADD(0, 1);
      if (spins > 1) __nanosleep(64);
#pragma unroll
      for (int c = 0; c < LBW; ++c)
        if ((uint32_t)(w[c] >> 32) != want) w[c] = dev::ld_relaxed_u64(P.status + base + lane + 32 * c);
    }
    uint32_t v = 0;
#pragma unroll
    for (int c = 0; c < LBW; ++c) v += (uint32_t)w[c];
    total += __reduce_add_sync(0xffffffffu, v);
  }
  return total;
}

// Compute warps: copy tile k's run of selected rows from the ring to its place
// (ROWS mode: the run holds row ids).
template <bool ROWS, typename SM>
__device__ __forceinline__ void write_tile(SM& S, const SelParams& P, int k, int tid) {
  // tell the look-back warp not to wait for later counts (a monotone hint,
  // relaxed accesses on both sides: never a plain racing access)
  if (tid == 0) st_relaxed_shared(&S.demand, k);
  PT_BEGIN(t0);
  mbar_wait(&S.placed[k % K], (uint32_t)((k / K) & 1));
  PT_END(2, t0, tid == 0);
  const int64_t g = S.goff[k % K];
  const int32_t c = S.cnt[k % K];
  if (ROWS && P.meta && tid == 0) *reinterpret_cast<int64_t*>(P.meta + S.tidx[k % K] * 12 + 8) = g;
  if (ROWS && !P.rowids) return;  // ids not requested: nothing in the ring
  const int32_t* run = S.ring + S.start[k % K];  // contiguous, never wraps
  int64_t lim = P.out_cap - g;
  lim = lim < 0 ? 0 : (lim > c ? c : lim);
  if (!ROWS) {
    int32_t* __restrict__ out = P.out + g;
    for (int e = tid; e < (int)lim; e += SEL_THREADS) out[e] = run[e];
  } else {
    uint32_t* __restrict__ out = P.rowids + g;
    for (int e = tid; e < (int)lim; e += SEL_THREADS) out[e] = (uint32_t)run[e];
  }
}

template <bool HAS_NE, bool ROWS>
__global__ void __launch_bounds__(BLOCK, 2) select_fused_kernel(const SelParams P) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  using SM = SelSmem;
  constexpr int RING = SM::kRing;
  SM& S = *reinterpret_cast<SM*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  // Programmatic dependent launch (launch_select_pass): this grid may start
  // while the previous kernel on the stream is finishing.  Nothing here reads
  // or writes global memory before the wait: the previous grid's results (its
  // output, count, epoch bump and ticket reset) are visible after it.
  dev::grid_dep_wait();
  if (tid == 0) {
    int64_t n = P.n;
    if (P.d_n) {
      const int64_t dn = dev::ld_relaxed_s64(P.d_n);
      n = dn < n ? (dn < 0 ? 0 : dn) : n;
    }
    S.n = n;
    S.epoch = ld_acquire_u32(&P.hdr[H_EPOCH]);  // advanced only by the last CTA out (epoch note above)
    S.demand = -1;
    S.sat = 0;
    for (int s = 0; s < SEL_INSLOTS; ++s) {
      mbar_init(&S.full[s], 1);
      mbar_init(&S.empty[s], 1);
    }
    for (int s = 0; s < Q; ++s) mbar_init(&S.winfull[s], 1);
    for (int s = 0; s < K; ++s) {
      mbar_init(&S.counted[s], 1);
      mbar_init(&S.placed[s], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int64_t n = S.n;
  const int64_t nv = n + P.mis;  // virtual rows, counted from the aligned base
  const int64_t ntiles = n > 0 ? (nv + SEL_TILE - 1) / SEL_TILE : 0;
  const uint64_t tag = S.epoch & TAG_MASK;

  if (warp == PRWARP) {
    // ======================= producer warp: partition + load ====================
    // Tickets are drawn one tile ahead of the slot they fill, so the atomic's L2
    // round trip overlaps the wait for that slot; a slot is refilled as soon as
    // the compute warps have read it (B1), giving up to SEL_INSLOTS tiles in flight.
    if (lane == 0) {
      // Tickets come in batches of G consecutive tiles; the next batch is drawn
      // as the current one starts, so an atomic's L2 round trip overlaps G
      // tiles of work.  G = 1 (measured, 2^28 rows: G = 2 is 2-4% faster at
      // overall selectivity <= .25 but 40% slower at .5/.9, where a drawn,
      // not yet counted tile holds up every later tile's placement; a second
      // single ticket drawn ahead only while the ring is under half full
      // gained nothing at .01/.25 and lost 5% at .5).
      constexpr int G = RA_SEL_BATCH;
      int64_t cur = (int64_t)atomicAdd(P.ticket, (unsigned long long)G);
      int64_t nxt = 0;
      int g = 0;
      for (int j = 0;; ++j) {
        const int s = j % SEL_INSLOTS;
        PT_BEGIN(t0);
        if (j >= SEL_INSLOTS) mbar_wait(&S.empty[s], (uint32_t)((j / SEL_INSLOTS - 1) & 1));
        PT_END(11, t0, true);
        if (g == G) {
          cur = nxt;
          g = 0;
        }
        const int64_t tn = cur + g;
        S.tile_of[s] = tn;
        if (tn >= ntiles) {  // end marker for the compute warps
          mbar_arrive(&S.full[s]);
          break;
        }
        issue_tile(S, P, nv, tn, s);
        if (g == 0) nxt = (int64_t)atomicAdd(P.ticket, (unsigned long long)G);
        ++g;
      }
    }
    return;
  }

  if (warp == LBWARP) {
    // ======================= look-back warp: tile offsets =======================
    const uint32_t want = (uint32_t)((FLAG_A | (tag << TAG_SHIFT)) >> 32);
    int64_t my_prefix = 0;  // inclusive prefix of this CTA's last placed tile
    int64_t t_last = -1;    // tile index of the last window copied
    int m = 0x7fffffff;     // tiles of this CTA, known once the end marker is counted
    // Decisions are warp-uniform: a lane that sees a barrier phase complete has
    // acquired it itself, and the warp acts only when all lanes agree.
    // tile x counted?  (and learn m from the end marker)
    auto counted = [&](int x) {
      if (x >= m) return true;
      if (!__all_sync(0xffffffffu, mbar_test(&S.counted[x % K], (uint32_t)((x / K) & 1)))) return false;
      if (S.tidx[x % K] < 0) m = x;
      return true;
    };
    // Tile k's window is copied once tile k+D1 is counted and resolved once
    // tile k+D2 is counted — or at once when the compute warps already wait
    // for tile k (`demand`: ring of selected rows full at high selectivity).
    auto due = [&](int k, int d) {
      return __all_sync(0xffffffffu, ld_relaxed_shared(&S.demand) >= k) || counted(k + d);
    };
    int c_next = 0;  // next window to copy
    for (int k = 0;; ++k) {
      PT_BEGIN(t0);
      mbar_wait(&S.counted[k % K], (uint32_t)((k / K) & 1));
      PT_END(9, t0, lane == 0);
      if (S.tidx[k % K] < 0) break;  // end marker
      for (int spins = 0;; ++spins) {
        if (c_next < k + Q && c_next < m && due(c_next, D1)) {
          // due(c, D1) implies tile c is counted; wait on it anyway to acquire tidx[]
          mbar_wait(&S.counted[c_next % K], (uint32_t)((c_next / K) & 1));
          const int64_t tc = S.tidx[c_next % K];
          if (tc < 0) {
            m = c_next;
          } else {
            if (lane == 0) issue_window(S, P, t_last + 1, tc, c_next % Q);
            t_last = tc;
            ++c_next;
          }
          continue;
        }
        if (c_next > k && due(k, D2)) break;
        if (spins > 2) __nanosleep(128);
      }
      {  // resolve tile k
        const int q = k % Q;
        PT_BEGIN(t0);
        mbar_wait(&S.winfull[q], (uint32_t)((k / Q) & 1));
        PT_END(6, t0, lane == 0);
        PT_BEGIN(t1);
        const int64_t g = my_prefix + window_sum(S, P, q, lane, want);
        PT_END(7, t1, lane == 0);
        const int64_t tp = S.whi[q];
        my_prefix = g + S.cnt[k % K];
        if (lane == 0) {
          S.goff[k % K] = g;
          // every later tile of this CTA has a larger index, so its offset is
          // >= my_prefix: in ROWS mode with my_prefix >= out_cap none of its
          // ids is written and the compute warps skip staging them
          if (ROWS && my_prefix >= P.out_cap) st_relaxed_shared(&S.sat, 1);
          if (tp == ntiles - 1) *P.d_count = my_prefix;  // every tile has published
          mbar_arrive(&S.placed[k % K]);
        }
        __syncwarp();
      }
    }
    // last CTA out resets the ticket counter for the next launch and advances
    // the epoch (after every CTA of this launch read it: one tag per launch)
    if (lane == 0) {
      __threadfence();
      if (atomicAdd(&P.hdr[H_DONE], 1u) == gridDim.x - 1) {
        *P.ticket = 0ull;
        P.hdr[H_DONE] = 0u;
        if (ntiles == 0) *P.d_count = 0;
        // High-water mark of status words this workspace has carried.  When the
        // next launch's 28-bit tag wraps to 0, clear all of them: a word left by
        // a launch exactly 2^28 launches earlier could otherwise read as ready.
        // (Every CTA of this launch is done with the status words; the next
        // launch reads them only after this grid completes.)
        uint64_t* hwm = reinterpret_cast<uint64_t*>(P.hdr + H_HWM);
        uint64_t h = *hwm;
        if ((uint64_t)ntiles > h) *hwm = h = (uint64_t)ntiles;
        if (((S.epoch + 1) & TAG_MASK) == 0)
          for (uint64_t w = 0; w < h; ++w) P.status[w] = 0ull;
        st_release_u32(&P.hdr[H_EPOCH], S.epoch + 1);
      }
    }
    return;
  }

  // ======================= compute warps ======================================
  int32_t wp = 0;    // end of the newest run in the ring
  int32_t used = 0;  // selected rows of pending tiles in the ring
  int head = 0;      // oldest tile not yet written
  int i = 0;
  PT_BEGIN(tloop);
  for (;; ++i) {
    const int slot = i % SEL_INSLOTS;
    PT_BEGIN(tf);
    mbar_wait(&S.full[slot], (uint32_t)((i / SEL_INSLOTS) & 1));
    PT_END(1, tf, tid == 0);
    PT_END(8, tf, tid == 224);
    const int64_t t = S.tile_of[slot];
    if (t >= ntiles) break;
    // ---- filter tile t
    int4 v[SEL_VEC];
    {
      const int4* base = &S.in[slot][warp * (WROWS / 4)];
#pragma unroll
      for (int j = 0; j < SEL_VEC; ++j) v[j] = base[32 * j + lane];
    }
    const int64_t v0 = t * SEL_TILE + warp * WROWS;
    uint32_t fl = 0;  // bit 4j+c: row warp*1024 + 4*(32j + lane) + c selected
    if (v0 >= P.mis && v0 + WROWS <= nv) {
#pragma unroll
      for (int j = 0; j < SEL_VEC; ++j)
#pragma unroll
        for (int c = 0; c < 4; ++c) fl |= (uint32_t)keep<HAS_NE>(comp(v[j], c), P) << (4 * j + c);
    } else {
#pragma unroll
      for (int j = 0; j < SEL_VEC; ++j) {
        const int64_t e0 = v0 + 4 * (32 * j + lane);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const bool in = (e0 + c >= P.mis) & (e0 + c < nv);
          fl |= (uint32_t)(keep<HAS_NE>(comp(v[j], c), P) & in) << (4 * j + c);
        }
      }
    }
    if (ROWS && P.fmask) P.fmask[t * SEL_THREADS + tid] = fl;  // for the payload compaction
    // ---- buffer: order (warp, j, lane, c); packed per-j counts, warp scans.
    // SWAR popcount of each nibble of fl (nibble j = the lane's 4 rows of
    // vector j), then j goes to word j&1, byte j>>1 (8 bits: a warp total <= 128).
    uint32_t packed[NPK], inc[NPK], tot[NPK];
    {
      uint32_t x = fl - ((fl >> 1) & 0x55555555u);
      x = (x & 0x33333333u) + ((x >> 2) & 0x33333333u);
      if (NPK == 2) {  // even j in word 0, odd j in word 1, byte j >> 1
        packed[0] = x & 0x0F0F0F0Fu;
        packed[NPK - 1] = (x >> 4) & 0x0F0F0F0Fu;
      } else {  // 16 flag bits: bytes j0, j2, j1, j3
        packed[0] = (x & 0x0F0Fu) | (((x >> 4) & 0x0F0Fu) << 16);
      }
#pragma unroll
      for (int q = 0; q < NPK; ++q) inc[q] = packed[q];
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
      for (int q = 0; q < NPK; ++q) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc[q], d);
        if (lane >= d) inc[q] += y;
      }
    }
    uint32_t wtotal = 0;
#pragma unroll
    for (int q = 0; q < NPK; ++q) {
      tot[q] = __shfl_sync(0xffffffffu, inc[q], 31);  // per-row warp totals (<= 128 each)
      wtotal += (tot[q] & 0xFF) + ((tot[q] >> 8) & 0xFF) + ((tot[q] >> 16) & 0xFF) + (tot[q] >> 24);
    }
    if (lane == 0) S.wtot[i & 1][warp] = wtotal;
    if (ROWS && tid == 0) S.past[i & 1] = (uint32_t)ld_relaxed_shared(&S.sat);  // one value for every thread
    PT_BEGIN(tb);
    compute_bar();  // B1: wtot visible; every warp is done with this tile's input slot
    PT_END(3, tb, tid == 0);
    PT_END(13, tb, tid == 224);
    const uint32_t wt = lane < NW ? S.wtot[i & 1][lane] : 0u;
    const int32_t agg = (int32_t)__reduce_add_sync(0xffffffffu, wt);
    const int32_t wbase = (int32_t)__reduce_add_sync(0xffffffffu, lane < warp ? wt : 0u);
    if (ROWS && P.meta && lane == 0) P.meta[t * 12 + warp] = (uint32_t)wbase;
    // ROWS without ids, or with every id of this tile past out_cap: no ring rows
    const bool ring_rows = !ROWS || (P.rowids && !S.past[i & 1]);
    const int32_t rows_in = ring_rows ? agg : 0;  // ring rows this tile needs
    if (tid == 0) {  // publish at once (before any wait below); hand the tile to the look-back warp
      S.rin[i % K] = rows_in;
      mbar_arrive(&S.empty[slot]);  // input slot free: the producer refills it
      dev::st_relaxed_u64(P.status + t, FLAG_A | (tag << TAG_SHIFT) | (uint64_t)agg);
      S.cnt[i % K] = agg;
      S.tidx[i % K] = t;
      mbar_arrive(&S.counted[i % K]);
    }
    // ---- allocate the tile's run: contiguous in the ring (a run that does not
    // fit before the end starts again at 0); write the oldest tiles early if
    // the ring is short.  Every thread takes the same decisions.
    int32_t start = 0;
    bool forced = false;
    while (true) {
      if (used == 0) {  // nothing pending (or only empty runs)
        start = 0;
        break;
      }
      // pending rows occupy [rp, wp), or [rp, end) + [0, wp) once they wrapped
      const int32_t rp = S.start[head % K];
      const bool wrapped = rp > wp || (rp == wp && used > 0);
      if (!wrapped) {
        if (wp + rows_in <= RING) { start = wp; break; }
        if (rows_in <= rp) { start = 0; break; }
      } else if (wp + rows_in <= rp) {
        start = wp;
        break;
      }
      write_tile<ROWS, SM>(S, P, head, tid);
      used -= S.rin[head % K];
      ++head;
      forced = true;
    }
    if (forced) compute_bar();  // rows written out are read before they are overwritten
    if (tid == 0) S.start[i % K] = start;
    used += rows_in;
    // ---- scatter the tile into the ring
    if (ring_rows) {
      int32_t rb = start + wbase;
#if RA_SEL_PTXSCATTER
      const uint32_t ring0 = smem_u32(S.ring);
#endif
#pragma unroll
      for (int j = 0; j < SEL_VEC; ++j) {
        const int q = q_of(j);
        const uint32_t ex = inc[q] - packed[q];
        int32_t p = rb + (int32_t)((ex >> (8 * b_of(j))) & 0xFFu);
#if RA_SEL_PTXSCATTER
        uint32_t a = ring0 + 4u * (uint32_t)p;  // byte address: one predicated store + add per row
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          // ROWS: the row id (n < 2^32 is checked by ra_select_rows)
          const int32_t val = ROWS ? (int32_t)(uint32_t)(t * SEL_TILE + warp * WROWS - P.mis + 4 * (32 * j + lane) + c)
                                   : comp(v[j], c);
          put_if(a, fl, 1u << (4 * j + c), val);
        }
#else
        const uint32_t bits = (fl >> (4 * j)) & 0xFu;
#pragma unroll
        for (int c = 0; c < 4; ++c)
          if (bits & (1u << c))
            S.ring[p++] = ROWS ? (int32_t)(uint32_t)(t * SEL_TILE + warp * WROWS - P.mis + 4 * (32 * j + lane) + c)
                               : comp(v[j], c);
#endif
        rb += (int32_t)((tot[q] >> (8 * b_of(j))) & 0xFFu);
      }
    }
    wp = start + rows_in;
    // ---- gather: tile i - LAG is due
    if (i - LAG >= head) {
      write_tile<ROWS, SM>(S, P, head, tid);
      used -= S.rin[head % K];
      ++head;
    }
  }
  PT_END(4, tloop, tid == 0);
  PROF_ADD(5, tid == 0 ? i : 0);
  if (tid == 0) {  // end marker for the look-back warp
    S.tidx[i % K] = -1;
    mbar_arrive(&S.counted[i % K]);
  }
  compute_bar();  // scatters of the last tiles are visible
  for (; head < i; ++head) write_tile<ROWS, SM>(S, P, head, tid);
}

// smem opt-in + occupancy of each instantiation, once per device
template <bool HAS_NE, bool ROWS>
int ensure_config(int dev, int& per_sm) {
  static std::atomic<int> cfg[64];
  const int v = device_once(cfg, dev, [] {
    const int smem = (int)sizeof(SelSmem);
    cudaError_t e = cudaFuncSetAttribute(select_fused_kernel<HAS_NE, ROWS>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(select smem)");
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, select_fused_kernel<HAS_NE, ROWS>, BLOCK, smem);
    if (e != cudaSuccess) return cuda_fail(e, "occupancy(select)");
    if (occ < 1) return fail(RA_E_CUDA, "select kernel does not fit on an SM");
    return occ;
  });
  if (v < 0) return v;
  per_sm = v;
  return RA_OK;
}

}  // namespace

int64_t sel_max_tiles(int64_t n) { return (n + 3 + SEL_TILE - 1) / SEL_TILE + 1; }

size_t sel_status_bytes(int64_t n) { return SEL_HDR_BYTES + 8 * (size_t)sel_max_tiles(n) + 16; }

size_t sel_inter_bytes(int64_t n) {
  // two int32[n] relations + two int64 counts, 256-B granules
  const size_t rel = (((size_t)(n > 0 ? n : 1) * 4 + 255) / 256) * 256;
  return 2 * rel + 256;
}

int sel_ctas_per_sm() {
  const int dev = current_device();
  int per_sm = 0;
  if (ensure_config<false, false>(dev, per_sm)) return -1;
  return per_sm;
}

int launch_select_pass(const int32_t* d_in, int64_t n_max, const int64_t* d_n, const CanonPred& cp,
                       int32_t* d_out, int64_t out_cap, int64_t* d_count, void* d_ws,
                       cudaStream_t s, uint32_t* rows, const SelMasks* masks) {
  SelParams P;
  P.rowids = rows;
  P.fmask = masks ? masks->fmask : nullptr;
  P.meta = masks ? masks->meta : nullptr;
  const uintptr_t a = (uintptr_t)d_in;
  P.mis = (int32_t)((a & 15u) >> 2);
  P.abase = (const int32_t*)(a - (a & 15u));
  P.n = n_max;
  P.d_n = d_n;
  P.out = d_out;
  P.out_cap = out_cap;
  P.d_count = d_count;
  P.hdr = (uint32_t*)d_ws;
  P.ticket = (unsigned long long*)((char*)d_ws + 8);
  P.status = (uint64_t*)((char*)d_ws + SEL_HDR_BYTES);
  P.lo = cp.lo;
  P.span = (uint32_t)cp.hi - (uint32_t)cp.lo;
  P.n_ne = cp.n_ne;
  for (int j = 0; j < RA_MAX_PREDS; ++j) P.ne[j] = j < cp.n_ne ? cp.ne[j] : 0;
  if (cp.lo > cp.hi) {  // empty interval: x == 0 and x != 0
    P.lo = 0;
    P.span = 0;
    P.n_ne = 1;
    P.ne[0] = 0;
  }
  if (n_max >= ((int64_t)1 << 34)) return fail(RA_E_INVAL, "n=%lld >= 2^34", (long long)n_max);
  const int dev = current_device();
  const bool ne = P.n_ne > 0;
  const bool rw = rows != nullptr || masks != nullptr;
  int per_sm = 1;
  int rc;
  const void* kern;
  if (rw) {
    rc = ne ? ensure_config<true, true>(dev, per_sm) : ensure_config<false, true>(dev, per_sm);
    kern = ne ? (const void*)select_fused_kernel<true, true> : (const void*)select_fused_kernel<false, true>;
  } else {
    rc = ne ? ensure_config<true, false>(dev, per_sm) : ensure_config<false, false>(dev, per_sm);
    kern = ne ? (const void*)select_fused_kernel<true, false> : (const void*)select_fused_kernel<false, false>;
  }
  if (rc) return rc;
  const int64_t ntiles_max = n_max > 0 ? (n_max + P.mis + SEL_TILE - 1) / SEL_TILE : 0;
  int64_t grid = (int64_t)num_sms() * per_sm;
  // RA_SEL_MAX_CTAS (diagnostics only): cap the grid, for the paper's Fig 12
  // experiment (a SELECT with half the CTAs, two of them on two streams)
  static const int64_t max_ctas = getenv("RA_SEL_MAX_CTAS") ? atoll(getenv("RA_SEL_MAX_CTAS")) : 0;
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
  if (grid > ntiles_max) grid = ntiles_max;
  if (grid < 1) grid = 1;
  // No co-residency is required (plain launch): a CTA only ever waits on the
  // aggregates of tiles with lower tickets, tickets are drawn only by running
  // CTAs, and a tile's aggregate is published before its CTA can block on
  // any placement — so the lowest unpublished tile can always be published.
  const size_t smem = sizeof(SelSmem);
  void* args[] = {(void*)&P};
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(BLOCK);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;  // overlap this launch with the previous
  attr[0].val.programmaticStreamSerializationAllowed = RA_SEL_PDL;   // kernel's tail (griddepcontrol.wait)
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t le = cudaLaunchKernelExC(&cfg, kern, args);
  if (le != cudaSuccess) return cuda_fail(le, "select_fused_kernel launch");
  count_launch();
  return RA_OK;
}

int select_chain_impl(const int32_t* d_in, int64_t n, const ra_pred* h_preds, int k, int fused,
                      int32_t* d_out, int64_t out_cap, int64_t* d_count, void* d_ws,
                      size_t ws_bytes, cudaStream_t s) {
  static const int64_t small_rows =
      getenv("RA_SEL_SMALL_ROWS") ? atoll(getenv("RA_SEL_SMALL_ROWS")) : RA_SEL_SMALL_ROWS_DEFAULT;
  if (fused || k <= 1) {
    // the fused chain is one output of the warp-specialised multi-output pass
    // (select_multi.cu): one kernel, writer warps, cooperative look-back.
    // Small inputs (a few tiles per SM) are launch/latency-bound: the lighter
    // single-output kernel of this file starts faster there (both produce the
    // same result; same workspace layout for one output).  RA_SEL_SMALL_ROWS
    // (diagnostics) moves the threshold.
    CanonPred cp;
    int rc = canonicalize(h_preds, k, &cp);
    if (rc) return rc;
    if (n <= small_rows) return launch_select_pass(d_in, n, nullptr, cp, d_out, out_cap, d_count, d_ws, s, nullptr);
    return launch_select_multi(d_in, n, &cp, 1, &d_out, &out_cap, &d_count, d_ws, s);
  }
  // Unfused composition: one pass per predicate, intermediates at the end of
  // the workspace (disjoint from any status words this workspace can hold).
  // (from the 256-B aligned end: a caller may pass any ws_bytes >= the required size)
  const size_t rel = (((size_t)(n > 0 ? n : 1) * 4 + 255) / 256) * 256;
  char* inter = (char*)d_ws + (ws_bytes & ~(size_t)255) - sel_inter_bytes(n);
  int32_t* buf[2] = {(int32_t*)inter, (int32_t*)(inter + rel)};
  int64_t* cnt = (int64_t*)(inter + 2 * rel);
  const int32_t* src = d_in;
  const int64_t* src_n = nullptr;
  for (int j = 0; j < k; ++j) {
    CanonPred cp;
    int rc = canonicalize(&h_preds[j], 1, &cp);
    if (rc) return rc;
    const bool last = (j == k - 1);
    int32_t* dst = last ? d_out : buf[j & 1];
    int64_t* dcnt = last ? d_count : &cnt[j & 1];
    // each pass is the same SELECT machinery as the fused chain (the
    // multi-output pass above the small-input threshold), so the fused /
    // unfused comparison measures fusion, not two kernel designs
    int64_t cap = last ? out_cap : n;
    rc = n <= small_rows ? launch_select_pass(src, n, src_n, cp, dst, cap, dcnt, d_ws, s, nullptr)
                         : launch_select_multi(src, n, &cp, 1, &dst, &cap, &dcnt, d_ws, s, src_n);
    if (rc) return rc;
    src = dst;
    src_n = dcnt;
  }
  return RA_OK;
}

}  // namespace ra
