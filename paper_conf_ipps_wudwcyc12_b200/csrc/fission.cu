// fission.cu — kernel fission for a host-resident SELECT chain (§IV).
//
// The paper's Stream Pool (Table IV) hands out CUDA
// streams and per-stream command lists; fission partitions a kernel into
// segments whose PCIe transfers overlap the computation of other segments
// (Fig 13), and a fused kernel under fission needs a CPU gather
// because "data is transferred to the CPU at different times" (§IV-C,
// L1456-1468).  This runner is that pool specialised to one pipeline:
//
//   chunk c -> stream c mod S:  H2D(chunk c)  ->  select_fused(chunk c)
//           -> count written straight into pinned h_chunk_counts[c] (mapped)
//   host, once chunk c's kernel event fires: D2H of exactly count_c values
//           into h_out + running offset  (the CPU gather as placement)
//
// The host waits on chunk c only when it is about to reuse chunk c's stream
// buffers (S chunks later), so S-1 H2D copies stay queued ahead of it and the
// copy engines never idle on a host round trip.

#include <stdio.h>
#include <string.h>

#include <vector>

#include "ra_internal.cuh"

namespace ra {

namespace {

size_t round256(size_t b) { return (b + 255) / 256 * 256; }

size_t per_stream_bytes(int64_t chunk_rows, int k, int fused) {
  const size_t io = round256((size_t)chunk_rows * 4);
  return 2 * io + round256(ra_select_workspace_bytes(chunk_rows, k, fused));
}

int check_pinned(const void* p, const char* name, void** dev_alias) {
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(RA_E_NOT_PINNED, "%s: not a CUDA-registered host pointer", name);
  }
  if (a.type != cudaMemoryTypeHost) return fail(RA_E_NOT_PINNED, "%s is not page-locked host memory", name);
  if (dev_alias) {
    *dev_alias = a.devicePointer;
    if (!*dev_alias) return fail(RA_E_NOT_PINNED, "%s has no device mapping", name);
  }
  return RA_OK;
}

}  // namespace

}  // namespace ra

using namespace ra;

RA_API size_t ra_fission_workspace_bytes(int64_t chunk_rows, int n_streams, int k, int fused) {
  if (chunk_rows <= 0 || n_streams <= 0) return 0;
  return (size_t)n_streams * per_stream_bytes(chunk_rows, k, fused);
}

RA_API int ra_fission_run(const int32_t* h_in, int64_t n, const ra_pred* h_preds, int k, int fused,
                          int64_t chunk_rows, const ra_stream_t* streams, int n_streams,
                          int32_t* h_out, int64_t out_cap, int64_t* h_count,
                          int64_t* h_chunk_counts, void* d_ws, size_t ws_bytes) {
  clear_error();
  if (n < 0 || k < 0 || k > RA_MAX_PREDS || chunk_rows <= 0 || n_streams <= 0 || out_cap < 0)
    return fail(RA_E_INVAL, "bad sizes (n=%lld k=%d chunk_rows=%lld n_streams=%d)", (long long)n, k,
                (long long)chunk_rows, n_streams);
  if (!h_count || !streams || (k > 0 && !h_preds)) return fail(RA_E_INVAL, "null argument");
  if (n > 0 && (!h_in || !h_chunk_counts || !d_ws || (out_cap > 0 && !h_out)))
    return fail(RA_E_INVAL, "null buffer with n > 0");
  if (((uintptr_t)h_in | (uintptr_t)h_out) & 3u) return fail(RA_E_INVAL, "host buffers must be 4-byte aligned");
  CanonPred cp;
  for (int j = 0; j < k; ++j) {
    int rc = canonicalize(&h_preds[j], 1, &cp);
    if (rc) return rc;
  }
  if (n == 0) {
    *h_count = 0;
    return RA_OK;
  }
  if (chunk_rows > n) chunk_rows = n;
  const size_t need = ra_fission_workspace_bytes(chunk_rows, n_streams, k, fused);
  if (ws_bytes < need)
    return fail(RA_E_WORKSPACE, "fission workspace %zu < required %zu", ws_bytes, need);
  int rc = check_pinned(h_in, "h_in", nullptr);
  if (rc) return rc;
  if (out_cap > 0 && (rc = check_pinned(h_out, "h_out", nullptr))) return rc;
  void* counts_alias = nullptr;
  if ((rc = check_pinned(h_chunk_counts, "h_chunk_counts", &counts_alias))) return rc;
  int64_t* d_counts = (int64_t*)counts_alias;

  const int S = n_streams;
  const size_t per = per_stream_bytes(chunk_rows, k, fused);
  const size_t io = round256((size_t)chunk_rows * 4);
  std::vector<cudaEvent_t> ev(S);
  for (int s = 0; s < S; ++s) {
    cudaError_t e = cudaEventCreateWithFlags(&ev[s], cudaEventDisableTiming);
    if (e != cudaSuccess) {
      for (int j = 0; j < s; ++j) cudaEventDestroy(ev[j]);
      return cuda_fail(e, "cudaEventCreate");
    }
  }
  // The per-stream select workspaces move with chunk_rows: re-zero their
  // control words (header + status, a few KB) so earlier calls' data in this
  // workspace can never read as tile status.
  for (int s = 0; s < S; ++s) {
    char* base = (char*)d_ws + (size_t)s * per;
    cudaError_t e = cudaMemsetAsync(base + 2 * io, 0, ra_select_workspace_bytes(chunk_rows, 1, 1),
                                    (cudaStream_t)streams[s]);
    if (e != cudaSuccess) {
      for (int j = 0; j < S; ++j) cudaEventDestroy(ev[j]);
      return cuda_fail(e, "cudaMemsetAsync(fission control words)");
    }
  }
  const int64_t C = (n + chunk_rows - 1) / chunk_rows;
  int64_t offset = 0;  // running output offset (CPU gather)
  int result = RA_OK;

  auto gather = [&](int64_t c) -> int {
    const int s = (int)(c % S);
    cudaError_t e = cudaEventSynchronize(ev[s]);
    if (e != cudaSuccess) return cuda_fail(e, "chunk event");
    const int64_t cnt = ((volatile int64_t*)h_chunk_counts)[c];
    int64_t ncopy = out_cap - offset;
    ncopy = ncopy < 0 ? 0 : (ncopy > cnt ? cnt : ncopy);
    if (ncopy > 0) {
      char* base = (char*)d_ws + (size_t)s * per;
      e = cudaMemcpyAsync(h_out + offset, base + io, (size_t)ncopy * 4, cudaMemcpyDeviceToHost,
                          (cudaStream_t)streams[s]);
      if (e != cudaSuccess) return cuda_fail(e, "D2H chunk result");
    }
    offset += cnt;
    return RA_OK;
  };

  for (int64_t c = 0; c < C && result == RA_OK; ++c) {
    const int s = (int)(c % S);
    if (c >= S && (result = gather(c - S)) != RA_OK) break;
    const int64_t r0 = c * chunk_rows;
    const int64_t len = (n - r0 < chunk_rows) ? (n - r0) : chunk_rows;
    char* base = (char*)d_ws + (size_t)s * per;
    int32_t* d_in = (int32_t*)base;
    int32_t* d_out = (int32_t*)(base + io);
    void* sel_ws = base + 2 * io;
    cudaStream_t st = (cudaStream_t)streams[s];
    cudaError_t e = cudaMemcpyAsync(d_in, h_in + r0, (size_t)len * 4, cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) {
      result = cuda_fail(e, "H2D chunk");
      break;
    }
    result = select_chain_impl(d_in, len, h_preds, k, fused, d_out, len, d_counts + c, sel_ws,
                               per - 2 * io, st);
    if (result != RA_OK) break;
    e = cudaEventRecord(ev[s], st);
    if (e != cudaSuccess) result = cuda_fail(e, "cudaEventRecord");
  }
  for (int64_t c = (C > S ? C - S : 0); c < C && result == RA_OK; ++c) result = gather(c);
  for (int s = 0; s < S; ++s) {
    cudaError_t e = cudaStreamSynchronize((cudaStream_t)streams[s]);
    if (e != cudaSuccess && result == RA_OK) result = cuda_fail(e, "stream sync");
    cudaEventDestroy(ev[s]);
  }
  if (result != RA_OK) return result;
  *h_count = offset;
  if (offset > out_cap)
    return fail(RA_E_CAPACITY, "%lld selected > out_cap %lld", (long long)offset, (long long)out_cap);
  return RA_OK;
}

// ------------------------------------------------------------------ Q1
namespace ra {
namespace {

// Per-stream region: the chunk's columns (each 256-B aligned), the Q1 kernel
// workspace and the stream's running partial.
struct Q1Region {
  size_t col[8];
  size_t ws, part, total;
};

Q1Region q1_region(int64_t chunk_rows, const size_t* esz, int ncol) {
  Q1Region r;
  size_t off = 0;
  for (int j = 0; j < ncol; ++j) {
    r.col[j] = off;
    off += round256((size_t)chunk_rows * esz[j]);
  }
  r.ws = off;
  r.part = r.ws + round256(q1_ws_bytes());
  r.total = r.part + round256(sizeof(ra_q1_partial));
  return r;
}

constexpr size_t WIDE_ESZ[7] = {4, 1, 1, 8, 8, 8, 8};    // ra_lineitem order
constexpr size_t NARROW_ESZ[6] = {2, 1, 2, 1, 1, 4};     // ra_lineitem_narrow order

// exact slotwise sum (the shard merge of ra_q1_finalize, without finalising)
void q1_merge(ra_q1_partial& acc, const ra_q1_partial& p) {
  acc.status |= p.status;
  acc.rows += p.rows;
  for (int s = 0; s < RA_Q1_GROUPS; ++s) {
    ra_q1_group& a = acc.group[s];
    const ra_q1_group& g = p.group[s];
    a.count += g.count;
    a.sum_qty += g.sum_qty;
    a.sum_base_price += g.sum_base_price;
    a.sum_disc += g.sum_disc;
    unsigned __int128 dp = ((unsigned __int128)(uint64_t)a.sum_disc_price_hi << 64) | a.sum_disc_price_lo;
    dp += ((unsigned __int128)(uint64_t)g.sum_disc_price_hi << 64) | g.sum_disc_price_lo;
    a.sum_disc_price_lo = (uint64_t)dp;
    a.sum_disc_price_hi = (int64_t)(uint64_t)(dp >> 64);
    unsigned __int128 ch = ((unsigned __int128)(uint64_t)a.sum_charge_hi << 64) | a.sum_charge_lo;
    ch += ((unsigned __int128)(uint64_t)g.sum_charge_hi << 64) | g.sum_charge_lo;
    a.sum_charge_lo = (uint64_t)ch;
    a.sum_charge_hi = (int64_t)(uint64_t)(ch >> 64);
  }
}

}  // namespace
}  // namespace ra

namespace ra {
namespace {

// Q1 under fission for any column layout: chunk c -> stream c % S: H2D of its
// column slices -> Q1 kernel accumulating into the stream's partial; the S
// partials are merged exactly at the end.  `launch(cols, len, partial, ws, st)`
// enqueues the layout's kernel in accumulate mode.
template <typename Launch>
int q1_fission_generic(const void* const* cols, const char* const* names, const size_t* esz, int ncol, int64_t n,
                       int64_t chunk_rows, const ra_stream_t* streams, int n_streams, ra_q1_partial* h_partial,
                       void* d_ws, size_t ws_bytes, Launch launch) {
  if (!h_partial || !streams) return fail(RA_E_INVAL, "null argument");
  if (n < 0 || n >= (int64_t)1 << 32 || chunk_rows <= 0 || n_streams <= 0)
    return fail(RA_E_INVAL, "bad sizes (n=%lld chunk_rows=%lld n_streams=%d)", (long long)n,
                (long long)chunk_rows, n_streams);
  memset(h_partial, 0, sizeof(*h_partial));
  h_partial->n_groups = RA_Q1_GROUPS;
  if (n == 0) return RA_OK;
  for (int j = 0; j < ncol; ++j)
    if (!cols[j]) return fail(RA_E_INVAL, "null column with n > 0");
  if (!d_ws) return fail(RA_E_INVAL, "null workspace");
  if ((uintptr_t)d_ws & 255u) return fail(RA_E_INVAL, "workspace must be 256-byte aligned");
  if (chunk_rows > n) chunk_rows = n;
  const Q1Region R = q1_region(chunk_rows, esz, ncol);
  const size_t need = (size_t)n_streams * R.total;
  if (ws_bytes < need) return fail(RA_E_WORKSPACE, "q1 fission workspace %zu < required %zu", ws_bytes, need);
  for (int j = 0; j < ncol; ++j) {
    int rc = check_pinned(cols[j], names[j], nullptr);
    if (rc) return rc;
  }
  const int S = n_streams;
  int result = RA_OK;
  // zero each stream's running partial and its Q1 ticket, status and grid
  // accumulators (the region
  // layout moves with chunk_rows)
  for (int s = 0; s < S && result == RA_OK; ++s) {
    char* base = (char*)d_ws + (size_t)s * R.total;
    cudaStream_t st = (cudaStream_t)streams[s];
    cudaError_t e = cudaMemsetAsync(base + R.part, 0, sizeof(ra_q1_partial), st);
    if (e == cudaSuccess) e = cudaMemsetAsync(base + R.ws, 0, q1_ws_clear_bytes(), st);
    if (e != cudaSuccess) result = cuda_fail(e, "cudaMemsetAsync(q1 fission partials)");
  }
  const int64_t C = (n + chunk_rows - 1) / chunk_rows;
  for (int64_t c = 0; c < C && result == RA_OK; ++c) {
    const int s = (int)(c % S);
    const int64_t r0 = c * chunk_rows;
    const int64_t len = (n - r0 < chunk_rows) ? (n - r0) : chunk_rows;
    char* base = (char*)d_ws + (size_t)s * R.total;
    cudaStream_t st = (cudaStream_t)streams[s];
    for (int j = 0; j < ncol && result == RA_OK; ++j) {
      cudaError_t e = cudaMemcpyAsync(base + R.col[j], (const char*)cols[j] + r0 * esz[j], (size_t)len * esz[j],
                                      cudaMemcpyHostToDevice, st);
      if (e != cudaSuccess) result = cuda_fail(e, "H2D q1 chunk column");
    }
    if (result != RA_OK) break;
    void* dcols[8];
    for (int j = 0; j < ncol; ++j) dcols[j] = base + R.col[j];
    result = launch(dcols, len, (ra_q1_partial*)(base + R.part), base + R.ws, st);
  }
  std::vector<ra_q1_partial> parts(S);
  for (int s = 0; s < S; ++s) {
    cudaStream_t st = (cudaStream_t)streams[s];
    if (result == RA_OK) {
      cudaError_t e = cudaMemcpyAsync(&parts[s], (char*)d_ws + (size_t)s * R.total + R.part,
                                      sizeof(ra_q1_partial), cudaMemcpyDeviceToHost, st);
      if (e != cudaSuccess) result = cuda_fail(e, "D2H q1 partial");
    }
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess && result == RA_OK) result = cuda_fail(e, "stream sync");
  }
  if (result != RA_OK) return result;
  for (int s = 0; s < S && s < C; ++s) q1_merge(*h_partial, parts[s]);
  h_partial->n_groups = RA_Q1_GROUPS;
  return RA_OK;
}

}  // namespace
}  // namespace ra

RA_API size_t ra_q1_fission_workspace_bytes(int64_t chunk_rows, int n_streams) {
  if (chunk_rows <= 0 || n_streams <= 0) return 0;
  return (size_t)n_streams * q1_region(chunk_rows, WIDE_ESZ, 7).total;
}

RA_API int ra_q1_fission_run(const ra_lineitem* h_cols, int64_t n, int32_t shipdate_cutoff,
                             int64_t chunk_rows, const ra_stream_t* streams, int n_streams,
                             ra_q1_partial* h_partial, void* d_ws, size_t ws_bytes) {
  clear_error();
  if (!h_cols) return fail(RA_E_INVAL, "null argument");
  const ra_lineitem& h = *h_cols;
  const void* cols[7] = {h.shipdate, h.returnflag, h.linestatus, h.quantity, h.extendedprice, h.discount, h.tax};
  static const char* const names[7] = {"shipdate", "returnflag", "linestatus", "quantity",
                                       "extendedprice", "discount", "tax"};
  return q1_fission_generic(cols, names, WIDE_ESZ, 7, n, chunk_rows, streams, n_streams, h_partial, d_ws, ws_bytes,
                            [&](void* const* d, int64_t len, ra_q1_partial* part, void* ws, cudaStream_t st) {
                              ra_lineitem c;
                              c.shipdate = (const int32_t*)d[0];
                              c.returnflag = (const uint8_t*)d[1];
                              c.linestatus = (const uint8_t*)d[2];
                              c.quantity = (const int64_t*)d[3];
                              c.extendedprice = (const int64_t*)d[4];
                              c.discount = (const int64_t*)d[5];
                              c.tax = (const int64_t*)d[6];
                              return launch_q1(c, len, shipdate_cutoff, part, ws, q1_ws_bytes(), st, 1);
                            });
}

RA_API size_t ra_q1_narrow_fission_workspace_bytes(int64_t chunk_rows, int n_streams) {
  if (chunk_rows <= 0 || n_streams <= 0) return 0;
  return (size_t)n_streams * q1_region(chunk_rows, NARROW_ESZ, 6).total;
}

RA_API int ra_q1_narrow_fission_run(const ra_lineitem_narrow* h_cols, int64_t n, int32_t shipdate_cutoff,
                                    int64_t chunk_rows, const ra_stream_t* streams, int n_streams,
                                    ra_q1_partial* h_partial, void* d_ws, size_t ws_bytes) {
  clear_error();
  if (!h_cols) return fail(RA_E_INVAL, "null argument");
  const ra_lineitem_narrow& h = *h_cols;
  const void* cols[6] = {h.shipdate, h.group, h.quantity, h.discount, h.tax, h.extendedprice};
  static const char* const names[6] = {"shipdate", "group", "quantity", "discount", "tax", "extendedprice"};
  return q1_fission_generic(cols, names, NARROW_ESZ, 6, n, chunk_rows, streams, n_streams, h_partial, d_ws,
                            ws_bytes,
                            [&](void* const* d, int64_t len, ra_q1_partial* part, void* ws, cudaStream_t st) {
                              ra_lineitem_narrow c;
                              c.shipdate = (const uint16_t*)d[0];
                              c.group = (const uint8_t*)d[1];
                              c.quantity = (const uint16_t*)d[2];
                              c.discount = (const uint8_t*)d[3];
                              c.tax = (const uint8_t*)d[4];
                              c.extendedprice = (const uint32_t*)d[5];
                              return launch_q1_narrow(c, len, shipdate_cutoff, part, ws, st, 1);
                            });
}
