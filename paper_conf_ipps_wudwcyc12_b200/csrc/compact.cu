// compact.cu — payload compaction of a tuple SELECT (ra_select_rows, SURVEY
// §8(f) f3): out_j[i] = col_j[row of the i-th selected tuple] for every payload
// field j, i < min(count, cap).
//
// The paper's SELECT ends with a gather of the selected rows (stage 4, Fig 3,
// PAPER.md L479-485).  For a multi-column relation the fused select pass over
// the key (select_fused.cu, ROWS mode) leaves, per 8192-row tile, the compute
// lanes' selection flag words, each compute warp's exclusive base within the
// tile and the tile's global output offset (SelMasks).  That is the complete
// order information: this kernel streams the payload columns tile by tile
// through a 3-stage shared-memory ring (one bulk async copy per tile and field
// plus the tile's 1 KB of flag words and 48-B record, issued by a producer
// warp), and each compute warp places the selected values of its 1024-row
// slice at
//     toff[t] + wbase[t][w] + (selected rows before it in the slice)
// using the same packed warp scan as the select kernel.  No ids, no look-back
// and no CTA barrier.  A field whose 16-B phase differs from the key's cannot
// be tile-copied in the key's row frame; its flagged elements are loaded from
// global memory directly.
#include "ra_internal.cuh"

namespace ra {
namespace {

constexpr int CT_WARPS = SEL_THREADS / 32;   // compute warps = select warps per tile (8)
constexpr int CT_BLOCK = SEL_THREADS + 32;   // + the producer warp
constexpr int CT_SLICE = SEL_TILE / CT_WARPS;   // rows per warp slice (1024)
constexpr int CT_STAGES = 3;  // x 2 CTAs per SM
constexpr int CT_STAGE_BYTES = SEL_TILE * 4;    // one tile of a 4-byte field, half a tile of an 8-byte one
static_assert(CT_SLICE == 32 * SEL_VEC * 4, "a slice is 32 lanes x SEL_VEC vectors x 4 rows");

struct CompactParams {
  const uint32_t* fmask;  // [tile][SEL_THREADS] flag words
  const uint32_t* meta;   // [tile][12]: wbase[8], int64 toff, pad
  const int64_t* d_count;
  int64_t n;      // rows
  int64_t cap;    // output capacity (elements)
  int32_t mis;    // rows of the key's 16-B chunk before row 0 (virtual rows = row + mis)
  int32_t m;
  int32_t sparse_den;
  const void* col[RA_MAX_PAYLOAD];
  void* out[RA_MAX_PAYLOAD];
  int32_t eb[RA_MAX_PAYLOAD];   // 4 or 8
  int32_t vec[RA_MAX_PAYLOAD];  // column phase matches the key's: tile copies
};

struct __align__(128) CtSmem {
  int4 data[CT_STAGES][CT_STAGE_BYTES / 16];
  uint32_t fl[CT_STAGES][SEL_THREADS];
  uint32_t meta[CT_STAGES][12];
  uint64_t full[CT_STAGES];
  uint64_t empty[CT_STAGES];
};

using dev::bulk_g2s;
using dev::mbar_arrive;
using dev::mbar_arrive_expect_tx;
using dev::mbar_init;
using dev::mbar_wait;

// Store v at a and advance a by one element, iff (fl & mask) != 0.
__device__ __forceinline__ void put_if_global(uint32_t*& a, uint32_t fl, uint32_t mask, uint32_t v) {
  asm volatile(
      "{\n\t.reg .pred q;\n\t.reg .b32 t;\n\t"
      "and.b32 t, %1, %2;\n\t"
      "setp.ne.u32 q, t, 0;\n\t"
      "@q st.global.b32 [%0], %3;\n\t"
      "@q add.u64 %0, %0, 4;\n\t}"
      : "+l"(a)
      : "r"(fl), "r"(mask), "r"(v)
      : "memory");
}
__device__ __forceinline__ void put_if_global(unsigned long long*& a, uint32_t fl, uint32_t mask,
                                              unsigned long long v) {
  asm volatile(
      "{\n\t.reg .pred q;\n\t.reg .b32 t;\n\t"
      "and.b32 t, %1, %2;\n\t"
      "setp.ne.u32 q, t, 0;\n\t"
      "@q st.global.b64 [%0], %3;\n\t"
      "@q add.u64 %0, %0, 8;\n\t}"
      : "+l"(a)
      : "r"(fl), "r"(mask), "l"(v)
      : "memory");
}

// The lane's exclusive (ex) and the warp's total (tot) packed counts of its
// flag word (as select_fused.cu): vector j's count at word j & 1, byte j >> 1.
__device__ __forceinline__ void packed_scan(uint32_t fl, int lane, uint32_t (&ex)[2], uint32_t (&tot)[2]) {
  uint32_t x = fl - ((fl >> 1) & 0x55555555u);  // nibble popcounts
  x = (x & 0x33333333u) + ((x >> 2) & 0x33333333u);
  const uint32_t pk[2] = {x & 0x0F0F0F0Fu, (x >> 4) & 0x0F0F0F0Fu};  // even j | odd j
  uint32_t inc[2] = {pk[0], pk[1]};
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc[q], d);
      if (lane >= d) inc[q] += y;
    }
  }
#pragma unroll
  for (int q = 0; q < 2; ++q) {
    ex[q] = inc[q] - pk[q];
    tot[q] = __shfl_sync(0xffffffffu, inc[q], 31);
  }
}

// Place the flagged elements of the lane's SEL_VEC vectors (rows of vector j:
// virtual vbase + 4*(32j + lane) + c) at out[dst0 + slice-local position].
template <typename T>
__device__ __forceinline__ void place(const CompactParams& P, int f, const int4* tile, int lane,
                                      int64_t vbase, uint32_t fl, int64_t dst0, int32_t lim,
                                      const uint32_t (&ex)[2], const uint32_t (&tot)[2]) {
  T* __restrict__ out = static_cast<T*>(P.out[f]) + dst0;
  constexpr int G = 32 / sizeof(T);  // vectors per batch (32 registers of elements)
  int32_t rb = 0;                    // slice-local output position
#pragma unroll
  for (int j0 = 0; j0 < SEL_VEC; j0 += G) {
    T e[G][4];
#pragma unroll
    for (int u = 0; u < G; ++u) {
      const int j = j0 + u;
      const uint32_t nib = (fl >> (4 * j)) & 0xFu;
      if (tile) {  // from the staged tile (warp slice = 1024 rows)
        if (sizeof(T) == 4) {
          const int4 v = tile[32 * j + lane];
          e[u][0] = (T)(uint32_t)v.x, e[u][1] = (T)(uint32_t)v.y, e[u][2] = (T)(uint32_t)v.z,
          e[u][3] = (T)(uint32_t)v.w;
        } else {
          const longlong2* t2 = reinterpret_cast<const longlong2*>(tile) + 2 * (32 * j + lane);
          const longlong2 a = t2[0], b = t2[1];
          e[u][0] = (T)a.x, e[u][1] = (T)a.y, e[u][2] = (T)b.x, e[u][3] = (T)b.y;
        }
      } else {  // phase mismatch: flagged elements from global memory
        const T* col = static_cast<const T*>(P.col[f]);
        const int64_t r = vbase + 4 * (32 * j + lane) - P.mis;
#pragma unroll
        for (int c = 0; c < 4; ++c) e[u][c] = (nib >> c) & 1u ? __ldg(col + r + c) : (T)0;
      }
    }
#pragma unroll
    for (int u = 0; u < G; ++u) {
      const int j = j0 + u;
      int32_t p = rb + (int32_t)((ex[j & 1] >> (8 * (j >> 1))) & 0xFFu);
      if (lim >= CT_SLICE) {  // the whole slice fits: one predicated store + add per row
        T* a = out + p;
#pragma unroll
        for (int c = 0; c < 4; ++c) put_if_global(a, fl, 1u << (4 * j + c), e[u][c]);
      } else {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          if ((fl >> (4 * j + c)) & 1u) {
            if (p < lim) out[p] = e[u][c];
            ++p;
          }
        }
      }
      rb += (int32_t)((tot[j & 1] >> (8 * (j >> 1))) & 0xFFu);
    }
  }
}

__global__ void __launch_bounds__(CT_BLOCK, 2) compact_kernel(const CompactParams P) {
  dev::grid_dep_wait();
  extern __shared__ __align__(128) unsigned char smem_raw[];
  CtSmem& S = *reinterpret_cast<CtSmem*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t nv = P.n + P.mis;
  const int64_t ntiles = (nv + SEL_TILE - 1) / SEL_TILE;
  int64_t cnt = *P.d_count;
  if (cnt * P.sparse_den <= P.n) return;  // sparse: gather_kernel places the fields (uniform exit)
  if (cnt > P.cap) cnt = P.cap;
  if (tid == 0) {
    for (int s = 0; s < CT_STAGES; ++s) {
      mbar_init(&S.full[s], 1);
      mbar_init(&S.empty[s], SEL_THREADS);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == CT_WARPS) {  // ---- producer: one unit = (tile, field)
    if (lane == 0) {
      int u = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int64_t v0 = t * SEL_TILE;
        const int64_t rows = nv - v0 < SEL_TILE ? nv - v0 : SEL_TILE;
        for (int f = 0; f < P.m; ++f)
        for (int h = 0; h < P.eb[f] / 4; ++h, ++u) {  // units: a 4-byte field's tile, or half an 8-byte one's
          const int s = u % CT_STAGES;
          if (u >= CT_STAGES) mbar_wait(&S.empty[s], (uint32_t)((u / CT_STAGES - 1) & 1));
          const int64_t h0 = (int64_t)h * (SEL_TILE / 2);  // first tile row of the unit (8-byte fields)
          const int64_t urows = P.eb[f] == 4 ? rows : (rows - h0 < SEL_TILE / 2 ? rows - h0 : SEL_TILE / 2);
          const uint32_t pb = P.vec[f] && urows > 0 ? (uint32_t)((urows * P.eb[f] + 15) & ~15ll) : 0u;
          // the key's 16-B aligned frame starts mis rows before the column; tile
          // 0 never reads before the column's own first 16-B granule (8-byte
          // fields with mis >= 2): the skipped rows are never flagged
          const char* base = static_cast<const char*>(P.col[f]) - (int64_t)P.mis * P.eb[f];
          const uint32_t skip = pb && t == 0 && h == 0 ? (uint32_t)(P.mis * P.eb[f]) & ~15u : 0u;
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          mbar_arrive_expect_tx(&S.full[s], pb - skip + SEL_THREADS * 4 + 48);
          if (pb)
            bulk_g2s(reinterpret_cast<char*>(&S.data[s][0]) + skip, base + (v0 + h0) * P.eb[f] + skip, pb - skip,
                     &S.full[s]);
          bulk_g2s(&S.fl[s][0], P.fmask + t * SEL_THREADS, SEL_THREADS * 4, &S.full[s]);
          bulk_g2s(&S.meta[s][0], P.meta + t * 12, 48, &S.full[s]);
        }
      }
    }
    return;
  }

  // ---- compute warps
  int u = 0;
  for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    for (int f = 0; f < P.m; ++f)
    for (int h = 0; h < P.eb[f] / 4; ++h, ++u) {
      const int s = u % CT_STAGES;
      mbar_wait(&S.full[s], (uint32_t)((u / CT_STAGES) & 1));
      const uint32_t fl = S.fl[s][tid];
      const int64_t dst0 = *reinterpret_cast<const int64_t*>(&S.meta[s][8]) + S.meta[s][warp];
      // 8-byte fields: unit h holds slices 4h..4h+3 (warps 4h..4h+3)
      const bool mine = P.eb[f] == 4 || (warp >> 2) == h;
      if (mine && __any_sync(0xffffffffu, fl != 0u) && dst0 < cnt) {
        const int32_t lim = cnt - dst0 < CT_SLICE ? (int32_t)(cnt - dst0) : CT_SLICE;
        uint32_t ex[2], tot[2];
        packed_scan(fl, lane, ex, tot);
        // the warp's slice in the staged unit
        const int4* tile = !P.vec[f] ? nullptr
                           : P.eb[f] == 4 ? &S.data[s][warp * (CT_SLICE / 4)] : &S.data[s][(warp & 3) * (CT_SLICE / 2)];
        const int64_t vbase = t * SEL_TILE + warp * CT_SLICE;
        if (P.eb[f] == 4)
          place<uint32_t>(P, f, tile, lane, vbase, fl, dst0, lim, ex, tot);
        else
          place<unsigned long long>(P, f, tile, lane, vbase, fl, dst0, lim, ex, tot);
      }
      mbar_arrive(&S.empty[s]);  // release-ordered after this thread's shared reads
    }
  }
}

// Sparse path, no ids from the key pass: ids[i] = row of the i-th selected
// tuple, from the order masks (one warp per 1024-row slice; predicated stores).
__global__ void __launch_bounds__(256) ids_kernel(const uint32_t* __restrict__ fmask, const uint32_t* __restrict__ meta,
                                                  const int64_t* __restrict__ d_count, int64_t n, int32_t mis,
                                                  int32_t sparse_den, int64_t staged, uint32_t* __restrict__ ids) {
  dev::grid_dep_wait();
  const int64_t cnt = *d_count;
  if (cnt * sparse_den > n) return;  // dense: compact_kernel places the fields, no ids needed
  if (cnt <= staged) return;         // the key pass staged them all
  const int lane = threadIdx.x & 31;
  const int64_t nslices = (n + mis + CT_SLICE - 1) / CT_SLICE;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x / 32);
  const int64_t w0 = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  constexpr int U = 4;  // slices per warp iteration: their loads are issued together
  for (int64_t sb = w0 * U; sb < nslices; sb += nw * U) {
    uint32_t fl[U];
    int64_t dst0[U];
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const int64_t sl = sb + q;
      fl[q] = sl < nslices ? __ldg(fmask + sl * 32 + lane) : 0u;
      const int64_t t = sl / CT_WARPS;
      dst0[q] = sl < nslices ? __ldg(reinterpret_cast<const long long*>(meta + t * 12 + 8)) +
                                   __ldg(meta + t * 12 + sl % CT_WARPS)
                             : 0;
    }
#pragma unroll
    for (int q = 0; q < U; ++q) {
      // a slice that ends before `staged` holds only ids the key pass wrote
      // (rewriting one it did write stores the same value)
      if (dst0[q] + CT_SLICE <= staged || !__any_sync(0xffffffffu, fl[q] != 0u)) continue;
      uint32_t ex[2], tot[2];
      packed_scan(fl[q], lane, ex, tot);
      const uint32_t r0 = (uint32_t)((sb + q) * CT_SLICE - mis);  // row of the slice's first virtual row (mod 2^32)
      uint32_t* a0 = ids + dst0[q];
      // one iteration per set bit b = 4j + c of the lane (the warp runs max
      // popcount iterations, ~1-3 on this sparse path; measured 1.5x faster
      // than a loop over the 8 vectors and their nibbles): its position is
      //   (warp's count in vectors j' < j) + (lanes < this one in vector j)
      //   + (this lane's bits below c in vector j)
      // the first term summed from the packed byte counts with dp4a.
      for (uint32_t f = fl[q]; f; f &= f - 1u) {
        const int b = __ffs(f) - 1, j = b >> 2;
        const uint32_t me = (uint32_t)((1ull << (8 * ((j + 1) >> 1))) - 1u);  // even j' < j: bytes [0, ceil(j/2))
        const uint32_t mo = (1u << (8 * (j >> 1))) - 1u;                       // odd j' < j: bytes [0, floor(j/2))
        const uint32_t pos = __dp4a(tot[0] & me, 0x01010101u, 0u) + __dp4a(tot[1] & mo, 0x01010101u, 0u) +
                             ((ex[j & 1] >> (8 * (j >> 1))) & 0xFFu) +
                             __popc(fl[q] & (0xFu << (4 * j)) & ((1u << b) - 1u));
        a0[pos] = r0 + 4 * (32 * j + lane) + (b & 3);
      }
    }
  }
}

}  // namespace

int launch_ids_from_masks(const int32_t* d_key, int64_t n, const SelMasks& mk, const int64_t* d_count,
                          int32_t sparse_den, int64_t staged, uint32_t* ids, cudaStream_t s) {
  if (n == 0) return RA_OK;
  const int32_t mis = (int32_t)(((uintptr_t)d_key & 15u) >> 2);
  const int64_t nslices = (n + mis + CT_SLICE - 1) / CT_SLICE;
  int64_t grid = (nslices + 31) / 32;  // 8 warps x 4 slices per CTA iteration
  const int64_t lim = (int64_t)num_sms() * 8;
  if (grid > lim) grid = lim;
  cudaError_t e = launch_pdl(ids_kernel, dim3((unsigned)grid), dim3(256), 0, s, (const uint32_t*)mk.fmask,
                             (const uint32_t*)mk.meta, d_count, n, mis, sparse_den, staged, ids);
  count_launch();
  if (e != cudaSuccess) return cuda_fail(e, "ids_kernel launch");
  return RA_OK;
}

size_t sel_masks_bytes(int64_t n) {
  const int64_t T = sel_max_tiles(n);
  return (size_t)T * (SEL_THREADS * 4 + 48) + 2 * 256;
}

int launch_compact(const int32_t* d_key, int64_t n, const SelMasks& mk, const int64_t* d_count, int64_t cap,
                   const GatherSpec& g, cudaStream_t s) {
  if (g.m == 0 || cap == 0 || n == 0) return RA_OK;
  static_assert(SEL_VEC == 8, "compact_kernel packs 8 vectors per lane");
  CompactParams P;
  P.fmask = mk.fmask;
  P.meta = mk.meta;
  P.d_count = d_count;
  P.n = n;
  P.cap = cap;
  P.mis = (int32_t)(((uintptr_t)d_key & 15u) >> 2);
  P.m = g.m;
  P.sparse_den = g.sparse_den;
  for (int j = 0; j < RA_MAX_PAYLOAD; ++j) {
    P.col[j] = j < g.m ? g.col[j] : nullptr;
    P.out[j] = j < g.m ? g.out[j] : nullptr;
    P.eb[j] = j < g.m ? g.elem_bytes[j] : 4;
    P.vec[j] = j < g.m && (((uintptr_t)g.col[j] - (uintptr_t)P.mis * (uintptr_t)g.elem_bytes[j]) & 15u) == 0;
  }
  static std::atomic<int> attr_set[64];
  const int a = device_once(attr_set, current_device(), [] {
    cudaError_t e = cudaFuncSetAttribute(compact_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sizeof(CtSmem));
    return e != cudaSuccess ? cuda_fail(e, "cudaFuncSetAttribute(compact smem)") : 1;
  });
  if (a < 0) return a;
  const int64_t ntiles = (n + P.mis + SEL_TILE - 1) / SEL_TILE;
  int64_t grid = (int64_t)num_sms() * 2;  // 2 CTAs per SM (launch bounds, ~100 KB of ring each)
  if (grid > ntiles) grid = ntiles;
  cudaError_t e = launch_pdl(compact_kernel, dim3((unsigned)grid), dim3(CT_BLOCK), sizeof(CtSmem), s, P);
  count_launch();
  if (e != cudaSuccess) return cuda_fail(e, "compact_kernel launch");
  return RA_OK;
}

}  // namespace ra
