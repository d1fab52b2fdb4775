// capi.cu — extern "C" entry points of libra.so (declared in include/ra.h):
// argument validation, workspace sizing, dispatch to the kernels, and the
// host-side Q1 finalize.  No allocation, no exceptions across the ABI.

#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "ra_internal.cuh"

namespace ra {

std::atomic<uint64_t> g_launches{0};

namespace {
thread_local char t_err[512] = "";
}

void clear_error() { t_err[0] = 0; }

int fail(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(t_err, sizeof(t_err), fmt, ap);
  va_end(ap);
  return code;
}

int cuda_fail(cudaError_t e, const char* what) {
  return fail(RA_E_CUDA, "%s: %s (%d)", what, cudaGetErrorString(e), (int)e);
}

std::mutex& init_mutex() {
  static std::mutex m;
  return m;
}

int current_device() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
  return dev;
}

int num_sms() {
  static std::atomic<int> cache[64];
  const int dev = current_device();
  return device_once(cache, dev, [&] {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    return v > 0 ? v : 148;
  });
}

int canonicalize(const ra_pred* preds, int k, CanonPred* out) {
  int32_t lo = INT32_MIN, hi = INT32_MAX;
  bool empty = false;
  int n_ne = 0;
  int32_t ne[RA_MAX_PREDS];
  for (int j = 0; j < k; ++j) {
    const int32_t v = preds[j].value;
    switch (preds[j].op) {
      case RA_LT:
        if (v == INT32_MIN) empty = true;
        else if (v - 1 < hi) hi = v - 1;
        break;
      case RA_LE:
        if (v < hi) hi = v;
        break;
      case RA_GT:
        if (v == INT32_MAX) empty = true;
        else if (v + 1 > lo) lo = v + 1;
        break;
      case RA_GE:
        if (v > lo) lo = v;
        break;
      case RA_EQ:
        if (v > lo) lo = v;
        if (v < hi) hi = v;
        break;
      case RA_NE: {
        bool dup = false;
        for (int i = 0; i < n_ne; ++i) dup |= (ne[i] == v);
        if (!dup) ne[n_ne++] = v;
        break;
      }
      default:
        return fail(RA_E_INVAL, "predicate %d: unknown op %d", j, (int)preds[j].op);
    }
  }
  if (empty || lo > hi) {
    lo = 1;
    hi = 0;  // empty interval
    n_ne = 0;
  }
  // drop exclusions outside the interval; an exclusion at an end shrinks it
  bool changed = true;
  while (changed && lo <= hi) {
    changed = false;
    for (int i = 0; i < n_ne; ++i) {
      if (ne[i] < lo || ne[i] > hi) {
        ne[i--] = ne[--n_ne];
        changed = true;
      } else if (ne[i] == lo && lo < hi) {
        lo = lo + 1;
        ne[i--] = ne[--n_ne];
        changed = true;
      } else if (ne[i] == hi && lo < hi) {
        hi = hi - 1;
        ne[i--] = ne[--n_ne];
        changed = true;
      } else if (lo == hi && ne[i] == lo) {
        lo = 1;
        hi = 0;
        n_ne = 0;
        changed = false;
        break;
      }
    }
  }
  out->lo = lo;
  out->hi = hi;
  out->n_ne = n_ne;
  for (int i = 0; i < RA_MAX_PREDS; ++i) out->ne[i] = i < n_ne ? ne[i] : 0;
  return RA_OK;
}

}  // namespace ra

using namespace ra;

RA_API const char* ra_last_error(void) { return t_err; }
RA_API int ra_version(void) { return 1; }
RA_API uint64_t ra_kernel_launches(void) { return g_launches.load(std::memory_order_relaxed); }

RA_API int ra_workspace_init(void* d_ws, size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  if (ws_bytes == 0) return RA_OK;
  if (!d_ws) return fail(RA_E_INVAL, "null workspace");
  cudaError_t e = cudaMemsetAsync(d_ws, 0, ws_bytes, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync(workspace)");
  return RA_OK;
}

RA_API size_t ra_select_workspace_bytes(int64_t n, int k, int fused) {
  if (n < 0) n = 0;
  // status words of either pass kind (the fused chain runs the multi-output
  // pass, the unfused composition's passes the single-output kernel)
  size_t b = (sel_status_bytes(n) + 255) / 256 * 256;
  if (ra::mo_workspace_bytes(n) > b) b = ra::mo_workspace_bytes(n);
  if (!fused && k > 1) b += sel_inter_bytes(n);
  return b;
}

static int check_select_args(const int32_t* d_in, int64_t n, int k, int32_t* d_out, int64_t out_cap,
                             int64_t* d_count, void* d_ws, size_t ws_bytes, int fused) {
  if (n < 0 || out_cap < 0) return fail(RA_E_INVAL, "negative n or out_cap");
  if (k < 0 || k > RA_MAX_PREDS) return fail(RA_E_INVAL, "k=%d outside [0, %d]", k, RA_MAX_PREDS);
  if (!d_count || !d_ws) return fail(RA_E_INVAL, "null d_count or workspace");
  if (n > 0 && !d_in) return fail(RA_E_INVAL, "null d_in with n > 0");
  if (out_cap > 0 && !d_out) return fail(RA_E_INVAL, "null d_out with out_cap > 0");
  if (((uintptr_t)d_in | (uintptr_t)d_out) & 3u) return fail(RA_E_INVAL, "pointers must be 4-byte aligned");
  if ((uintptr_t)d_count & 7u) return fail(RA_E_INVAL, "d_count must be 8-byte aligned");
  if ((uintptr_t)d_ws & 255u) return fail(RA_E_INVAL, "workspace must be 256-byte aligned");
  const size_t need = ra_select_workspace_bytes(n, k, fused);
  if (ws_bytes < need) return fail(RA_E_WORKSPACE, "workspace %zu < required %zu", ws_bytes, need);
  return RA_OK;
}

RA_API int ra_select(const int32_t* d_in, int64_t n, ra_pred pred, int32_t* d_out, int64_t out_cap,
                     int64_t* d_count, void* d_ws, size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  int rc = check_select_args(d_in, n, 1, d_out, out_cap, d_count, d_ws, ws_bytes, 1);
  if (rc) return rc;
  return select_chain_impl(d_in, n, &pred, 1, 1, d_out, out_cap, d_count, d_ws, ws_bytes,
                           (cudaStream_t)stream);
}

RA_API int ra_select_chain(const int32_t* d_in, int64_t n, const ra_pred* h_preds, int k, int fused,
                           int32_t* d_out, int64_t out_cap, int64_t* d_count, void* d_ws,
                           size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  int rc = check_select_args(d_in, n, k, d_out, out_cap, d_count, d_ws, ws_bytes, fused);
  if (rc) return rc;
  if (k > 0 && !h_preds) return fail(RA_E_INVAL, "null h_preds with k > 0");
  for (int j = 0; j < k; ++j)
    if (h_preds[j].op < RA_LT || h_preds[j].op > RA_NE)
      return fail(RA_E_INVAL, "predicate %d: unknown op %d", j, (int)h_preds[j].op);
  return select_chain_impl(d_in, n, h_preds, k, fused, d_out, out_cap, d_count, d_ws, ws_bytes,
                           (cudaStream_t)stream);
}

RA_API size_t ra_select_multi_workspace_bytes(int64_t n) {
  if (n < 0) n = 0;
  return ra::mo_workspace_bytes(n);
}

RA_API int ra_select_multi(const int32_t* d_in, int64_t n, const ra_pred* const* h_chains, const int* ks, int M,
                           int32_t* const* d_outs, const int64_t* out_caps, int64_t* const* d_counts, void* d_ws,
                           size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  if (M < 1 || M > RA_MAX_OUTPUTS) return fail(RA_E_INVAL, "M=%d outside [1, %d]", M, RA_MAX_OUTPUTS);
  if (!h_chains || !ks || !d_outs || !out_caps || !d_counts || !d_ws) return fail(RA_E_INVAL, "null argument");
  if (n < 0) return fail(RA_E_INVAL, "negative n");
  if (n > 0 && !d_in) return fail(RA_E_INVAL, "null d_in with n > 0");
  if ((uintptr_t)d_in & 3u) return fail(RA_E_INVAL, "d_in must be 4-byte aligned");
  if ((uintptr_t)d_ws & 255u) return fail(RA_E_INVAL, "workspace must be 256-byte aligned");
  const size_t need = ra_select_multi_workspace_bytes(n);
  if (ws_bytes < need) return fail(RA_E_WORKSPACE, "workspace %zu < required %zu", ws_bytes, need);
  CanonPred cp[RA_MAX_OUTPUTS];
  for (int o = 0; o < M; ++o) {
    if (out_caps[o] < 0) return fail(RA_E_INVAL, "output %d: negative out_cap", o);
    if (out_caps[o] > 0 && !d_outs[o]) return fail(RA_E_INVAL, "output %d: null d_out with out_cap > 0", o);
    if (!d_counts[o]) return fail(RA_E_INVAL, "output %d: null d_count", o);
    if (((uintptr_t)d_outs[o] & 3u) || ((uintptr_t)d_counts[o] & 7u))
      return fail(RA_E_INVAL, "output %d: misaligned d_out or d_count", o);
    if (ks[o] < 0 || ks[o] > RA_MAX_PREDS) return fail(RA_E_INVAL, "output %d: k=%d outside [0, %d]", o, ks[o], RA_MAX_PREDS);
    if (ks[o] > 0 && !h_chains[o]) return fail(RA_E_INVAL, "null chain %d with k > 0", o);
    for (int j = 0; j < ks[o]; ++j)
      if (h_chains[o][j].op < RA_LT || h_chains[o][j].op > RA_NE)
        return fail(RA_E_INVAL, "output %d predicate %d: unknown op %d", o, j, (int)h_chains[o][j].op);
    int rc = canonicalize(h_chains[o], ks[o], &cp[o]);
    if (rc) return rc;
  }
  return ra::launch_select_multi(d_in, n, cp, M, d_outs, out_caps, d_counts, d_ws, (cudaStream_t)stream);
}

RA_API size_t ra_select_rows_workspace_bytes(int64_t n, int k) {
  if (n < 0) n = 0;
  // select status words, then the per-tile masks for the payload compaction
  // (and, for the A/B against the id gather, a staging area for the row ids)
  return ((ra_select_workspace_bytes(n, k, 1) + 255) / 256) * 256 + ((ra::sel_masks_bytes(n) + 255) / 256) * 256 +
         (((size_t)n * 4 + 255) / 256) * 256;
}

#ifndef RA_TUPLE_STAGE_DEN
#define RA_TUPLE_STAGE_DEN 32  // without caller ids the key pass stages the first n/32 (A/B knob)
#endif

RA_API int ra_select_rows(const int32_t* d_key, int64_t n, const ra_pred* h_preds, int k, uint32_t* d_rowids,
                          const ra_payload* h_payloads, int m, int64_t out_cap, int64_t* d_count, void* d_ws,
                          size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  int rc = check_select_args(d_key, n, k, nullptr, 0, d_count, d_ws, ws_bytes, 1);
  if (rc) return rc;
  if (out_cap < 0) return fail(RA_E_INVAL, "negative out_cap");
  if (n >= (int64_t)1 << 32) return fail(RA_E_INVAL, "n=%lld >= 2^32 (row ids are uint32)", (long long)n);
  if (m < 0 || m > RA_MAX_PAYLOAD) return fail(RA_E_INVAL, "m=%d outside [0, %d]", m, RA_MAX_PAYLOAD);
  if (m > 0 && !h_payloads) return fail(RA_E_INVAL, "null h_payloads with m > 0");
  if (k > 0 && !h_preds) return fail(RA_E_INVAL, "null h_preds with k > 0");
  for (int j = 0; j < k; ++j)
    if (h_preds[j].op < RA_LT || h_preds[j].op > RA_NE)
      return fail(RA_E_INVAL, "predicate %d: unknown op %d", j, (int)h_preds[j].op);
  if ((uintptr_t)d_rowids & 3u) return fail(RA_E_INVAL, "d_rowids must be 4-byte aligned");
  const size_t need = ra_select_rows_workspace_bytes(n, k);
  if (ws_bytes < need) return fail(RA_E_WORKSPACE, "workspace %zu < required %zu", ws_bytes, need);
  GatherSpec g;
  g.m = m;
  g.n = n;
  g.sparse_den = 10;  // 4-byte fields: gather up to 1/10 selected (measured crossover)
  for (int j = 0; j < m; ++j) {
    const ra_payload& p = h_payloads[j];
    if (p.elem_bytes != 4 && p.elem_bytes != 8)
      return fail(RA_E_INVAL, "payload %d: elem_bytes %d not 4 or 8", j, (int)p.elem_bytes);
    if ((n > 0 && !p.col) || (out_cap > 0 && !p.out)) return fail(RA_E_INVAL, "payload %d: null column", j);
    if (((uintptr_t)p.col | (uintptr_t)p.out) & (uintptr_t)(p.elem_bytes - 1))
      return fail(RA_E_INVAL, "payload %d: pointers not %d-byte aligned", j, (int)p.elem_bytes);
    g.elem_bytes[j] = p.elem_bytes;
    g.col[j] = p.col;
    g.out[j] = p.out;
    if (p.elem_bytes == 8) g.sparse_den = 4;  // 8-byte fields: one gathered row moves 2x the bytes, crossover 1/4
  }
  CanonPred cp;
  rc = canonicalize(h_preds, k, &cp);
  if (rc) return rc;
  // Without caller ids the ids of the sparse path come from the key pass (the
  // first n/32, staged) and ids_kernel (the rest, from the order masks): the
  // crossover with the compaction is at a lower selectivity.
  if (!d_rowids) g.sparse_den = g.sparse_den == 4 ? 8 : 12;
  if (getenv("RA_TUPLE_GATHER")) g.sparse_den = 0;  // A/B only: always the id gather
  // One fused pass over the key writes the caller's row ids (if asked for) and
  // the per-tile order masks; then the payload fields are placed by the gather
  // (sparse; ids rebuilt from the masks into the workspace when the caller
  // did not ask for them) or by the streaming compaction (dense), chosen on
  // the device from the count.
  // masks and staged ids sit at the (256-B aligned) END of the workspace, so
  // the status words of a later call with any n never overlap them
  const size_t extra = ((ra::sel_masks_bytes(n) + 255) / 256) * 256 + (((size_t)n * 4 + 255) / 256) * 256;
  const size_t mask_off = (ws_bytes & ~(size_t)255) - extra;
  const size_t stage_off = mask_off + ((ra::sel_masks_bytes(n) + 255) / 256) * 256;
  uint32_t* ids = d_rowids ? d_rowids : (uint32_t*)((char*)d_ws + stage_off);
  const int64_t T = ra::sel_max_tiles(n);
  char* mb = (char*)d_ws + mask_off;
  ra::SelMasks mk;
  mk.fmask = (uint32_t*)mb;
  mk.meta = (uint32_t*)(mb + (((size_t)T * SEL_THREADS * 4 + 255) / 256) * 256);
  const bool masks = m > 0 && g.sparse_den > 0;
  // Staging ids in the key pass costs a dense call ~0.15 ms per n of ids (the
  // ring of selected rows fills and waits for the look-back), so only the
  // first n/32 are staged; a count up to that needs no ids_kernel at all.
  int64_t cap = d_rowids ? out_cap : (out_cap < n ? out_cap : n);
  if (!d_rowids && masks && cap > n / RA_TUPLE_STAGE_DEN) cap = n / RA_TUPLE_STAGE_DEN;
  rc = launch_select_pass(d_key, n, nullptr, cp, nullptr, cap, d_count, d_ws, (cudaStream_t)stream,
                          (d_rowids || m > 0) && cap > 0 ? ids : nullptr, masks ? &mk : nullptr);
  if (rc) return rc;
  if (masks && !d_rowids) {
    rc = ra::launch_ids_from_masks(d_key, n, mk, d_count, g.sparse_den, cap, ids, (cudaStream_t)stream);
    if (rc) return rc;
  }
  rc = launch_gather(ids, d_count, out_cap < n ? out_cap : n, g, (cudaStream_t)stream);
  if (rc || g.sparse_den == 0) return rc;
  return ra::launch_compact(d_key, n, mk, d_count, out_cap, g, (cudaStream_t)stream);
}

RA_API size_t ra_q1_workspace_bytes(int64_t n) {
  (void)n;
  return q1_ws_bytes();
}

RA_API int ra_q1(const ra_lineitem* h_cols, int64_t n, int32_t shipdate_cutoff, ra_q1_partial* d_partial,
                 void* d_ws, size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  if (!h_cols || !d_partial || !d_ws) return fail(RA_E_INVAL, "null argument");
  if (n < 0 || n >= (int64_t)1 << 32) return fail(RA_E_INVAL, "n=%lld outside [0, 2^32)", (long long)n);
  const ra_lineitem& c = *h_cols;
  if (n > 0 && (!c.shipdate || !c.returnflag || !c.linestatus || !c.quantity || !c.extendedprice ||
                !c.discount || !c.tax))
    return fail(RA_E_INVAL, "null column with n > 0");
  if (((uintptr_t)c.shipdate & 3u) || (((uintptr_t)c.quantity | (uintptr_t)c.extendedprice |
                                        (uintptr_t)c.discount | (uintptr_t)c.tax) & 7u))
    return fail(RA_E_INVAL, "columns must be naturally aligned");
  if ((uintptr_t)d_partial & 7u) return fail(RA_E_INVAL, "d_partial must be 8-byte aligned");
  if ((uintptr_t)d_ws & 255u) return fail(RA_E_INVAL, "workspace must be 256-byte aligned");
  if (ws_bytes < q1_ws_bytes()) return fail(RA_E_WORKSPACE, "workspace %zu < required %zu", ws_bytes, q1_ws_bytes());
  return launch_q1(c, n, shipdate_cutoff, d_partial, d_ws, ws_bytes, (cudaStream_t)stream);
}

RA_API int ra_q1_encode(const ra_lineitem* h_cols, int64_t n, const ra_lineitem_narrow_out* h_out,
                        uint32_t* d_status, ra_stream_t stream) {
  clear_error();
  if (!h_cols || !h_out || !d_status) return fail(RA_E_INVAL, "null argument");
  if (n < 0 || n >= (int64_t)1 << 32) return fail(RA_E_INVAL, "n=%lld outside [0, 2^32)", (long long)n);
  const ra_lineitem& c = *h_cols;
  const ra_lineitem_narrow_out& o = *h_out;
  if (n > 0 && (!c.shipdate || !c.returnflag || !c.linestatus || !c.quantity || !c.extendedprice ||
                !c.discount || !c.tax || !o.shipdate || !o.group || !o.quantity || !o.discount || !o.tax ||
                !o.extendedprice))
    return fail(RA_E_INVAL, "null column with n > 0");
  if (((uintptr_t)c.shipdate & 3u) || (((uintptr_t)c.quantity | (uintptr_t)c.extendedprice |
                                        (uintptr_t)c.discount | (uintptr_t)c.tax) & 7u))
    return fail(RA_E_INVAL, "input columns must be naturally aligned");
  if (((uintptr_t)o.shipdate | (uintptr_t)o.group | (uintptr_t)o.quantity | (uintptr_t)o.discount |
       (uintptr_t)o.tax | (uintptr_t)o.extendedprice) & 15u)
    return fail(RA_E_INVAL, "narrow columns must be 16-byte aligned");
  if ((uintptr_t)d_status & 3u) return fail(RA_E_INVAL, "d_status must be 4-byte aligned");
  return launch_q1_encode(c, n, o, d_status, (cudaStream_t)stream);
}

RA_API int ra_q1_narrow(const ra_lineitem_narrow* h_cols, int64_t n, int32_t shipdate_cutoff,
                        ra_q1_partial* d_partial, void* d_ws, size_t ws_bytes, ra_stream_t stream) {
  clear_error();
  if (!h_cols || !d_partial || !d_ws) return fail(RA_E_INVAL, "null argument");
  if (n < 0 || n >= (int64_t)1 << 32) return fail(RA_E_INVAL, "n=%lld outside [0, 2^32)", (long long)n);
  const ra_lineitem_narrow& c = *h_cols;
  if (n > 0 && (!c.shipdate || !c.group || !c.quantity || !c.discount || !c.tax || !c.extendedprice))
    return fail(RA_E_INVAL, "null column with n > 0");
  if (((uintptr_t)c.shipdate | (uintptr_t)c.group | (uintptr_t)c.quantity | (uintptr_t)c.discount |
       (uintptr_t)c.tax | (uintptr_t)c.extendedprice) & 15u)
    return fail(RA_E_INVAL, "narrow columns must be 16-byte aligned");
  if ((uintptr_t)d_partial & 7u) return fail(RA_E_INVAL, "d_partial must be 8-byte aligned");
  if ((uintptr_t)d_ws & 255u) return fail(RA_E_INVAL, "workspace must be 256-byte aligned");
  if (ws_bytes < q1_ws_bytes()) return fail(RA_E_WORKSPACE, "workspace %zu < required %zu", ws_bytes, q1_ws_bytes());
  return launch_q1_narrow(c, n, shipdate_cutoff, d_partial, d_ws, (cudaStream_t)stream);
}

RA_API int ra_q1_finalize(const ra_q1_partial* h_partials, int n_partials, ra_q1_row* h_rows, int* n_rows) {
  clear_error();
  if (n_partials < 0 || (n_partials > 0 && !h_partials) || !h_rows || !n_rows)
    return fail(RA_E_INVAL, "null argument");
  static const uint8_t RF[3] = {'A', 'N', 'R'}, LS[2] = {'F', 'O'};
  uint32_t status = 0;
  int m = 0;
  for (int s = 0; s < RA_Q1_GROUPS; ++s) {  // slot order == ORDER BY (rf, ls)
    int64_t cnt = 0, sq = 0, sp = 0, sd = 0;
    unsigned __int128 dp = 0, ch = 0;
    for (int i = 0; i < n_partials; ++i) {
      const ra_q1_group& g = h_partials[i].group[s];
      if (s == 0) status |= h_partials[i].status;
      cnt += g.count;
      sq += g.sum_qty;
      sp += g.sum_base_price;
      sd += g.sum_disc;
      dp += ((unsigned __int128)(uint64_t)g.sum_disc_price_hi << 64) | g.sum_disc_price_lo;
      ch += ((unsigned __int128)(uint64_t)g.sum_charge_hi << 64) | g.sum_charge_lo;
    }
    if (cnt == 0) continue;  // GROUP BY emits no empty groups
    ra_q1_row& r = h_rows[m++];
    memset(&r, 0, sizeof(r));
    r.returnflag = RF[s >> 1];
    r.linestatus = LS[s & 1];
    r.count_order = cnt;
    r.sum_qty = sq;
    r.sum_base_price = sp;
    r.sum_disc = sd;
    r.sum_disc_price_lo = (uint64_t)dp;
    r.sum_disc_price_hi = (int64_t)(uint64_t)(dp >> 64);
    r.sum_charge_lo = (uint64_t)ch;
    r.sum_charge_hi = (int64_t)(uint64_t)(ch >> 64);
    const double den = (double)(cnt * 100);  // one division of exact operands (C12)
    r.avg_qty = (double)sq / den;
    r.avg_price = (double)sp / den;
    r.avg_disc = (double)sd / den;
  }
  *n_rows = m;
  if (status) return fail(RA_E_DOMAIN, "Q1 input outside the domain (status 0x%x)", status);
  return RA_OK;
}
