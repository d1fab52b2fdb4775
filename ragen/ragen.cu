// ragen.cu — host (multithreaded) and device implementations of the seeded
// input generator in ragen_core.h.  INPUT GENERATION ONLY (see the header).
//
// Both sides evaluate the same integer-only functions, so host- and
// device-generated ranges are byte-identical (tests/test_ragen*.py).

#include <cuda_runtime.h>
#include <pthread.h>
#include <stdint.h>
#include <string.h>

#include "ragen_core.h"

#define RAGEN_API extern "C" __attribute__((visibility("default")))

// ---------------------------------------------------------------- host side
namespace {

struct HostJob {
  int kind;  // 0 = int32, 1 = lineitem
  uint64_t seed;
  uint32_t n_parts;
  uint64_t row0;
  int64_t lo, hi;  // local index range [lo, hi)
  int32_t* x;
  int32_t* shipdate;
  uint8_t* rf;
  uint8_t* ls;
  int64_t *qty, *ep, *disc, *tax;
};

void* host_worker(void* arg) {
  HostJob* j = (HostJob*)arg;
  if (j->kind == 0) {
    uint64_t key = ragen_key(j->seed, RAGEN_S_INT32);
    for (int64_t i = j->lo; i < j->hi; ++i) j->x[i] = ragen_int32_at(key, j->row0 + (uint64_t)i);
  } else {
    ragen_lineitem_keys k = ragen_lineitem_make_keys(j->seed, j->n_parts);
    for (int64_t i = j->lo; i < j->hi; ++i) {
      ragen_lineitem_row r = ragen_lineitem_at(&k, j->row0 + (uint64_t)i);
      if (j->shipdate) j->shipdate[i] = r.shipdate;
      if (j->rf) j->rf[i] = r.returnflag;
      if (j->ls) j->ls[i] = r.linestatus;
      if (j->qty) j->qty[i] = r.quantity;
      if (j->ep) j->ep[i] = r.extendedprice;
      if (j->disc) j->disc[i] = r.discount;
      if (j->tax) j->tax[i] = r.tax;
    }
  }
  return nullptr;
}

void run_host(HostJob base, int64_t n, int nthreads) {
  if (n <= 0) return;
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 256) nthreads = 256;
  if (n < (int64_t)nthreads * 65536) nthreads = (int)((n + 65535) / 65536);
  HostJob jobs[256];
  pthread_t th[256];
  for (int t = 0; t < nthreads; ++t) {
    jobs[t] = base;
    jobs[t].lo = n * t / nthreads;
    jobs[t].hi = n * (t + 1) / nthreads;
  }
  for (int t = 1; t < nthreads; ++t) pthread_create(&th[t], nullptr, host_worker, &jobs[t]);
  host_worker(&jobs[0]);
  for (int t = 1; t < nthreads; ++t) pthread_join(th[t], nullptr);
}

}  // namespace

// x[i] = int32 draw of global row (row0 + i), i in [0, n)
RAGEN_API void ragen_int32_host(uint64_t seed, uint64_t row0, int64_t n, int32_t* x, int nthreads) {
  HostJob j;
  memset(&j, 0, sizeof(j));
  j.kind = 0;
  j.seed = seed;
  j.row0 = row0;
  j.x = x;
  run_host(j, n, nthreads);
}

// Any column pointer may be NULL (not generated).
RAGEN_API void ragen_lineitem_host(uint64_t seed, uint32_t n_parts, uint64_t row0, int64_t n,
                                   int32_t* shipdate, uint8_t* returnflag, uint8_t* linestatus,
                                   int64_t* quantity, int64_t* extendedprice, int64_t* discount,
                                   int64_t* tax, int nthreads) {
  HostJob j;
  memset(&j, 0, sizeof(j));
  j.kind = 1;
  j.seed = seed;
  j.n_parts = n_parts;
  j.row0 = row0;
  j.shipdate = shipdate;
  j.rf = returnflag;
  j.ls = linestatus;
  j.qty = quantity;
  j.ep = extendedprice;
  j.disc = discount;
  j.tax = tax;
  run_host(j, n, nthreads);
}

// -------------------------------------------------------------- device side
namespace {

__global__ void k_int32(uint64_t key, uint64_t row0, int64_t n, int32_t* __restrict__ x) {
  int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
    x[i] = ragen_int32_at(key, row0 + (uint64_t)i);
}

__global__ void k_lineitem(ragen_lineitem_keys k, uint64_t row0, int64_t n, int32_t* shipdate,
                           uint8_t* rf, uint8_t* ls, int64_t* qty, int64_t* ep, int64_t* disc,
                           int64_t* tax) {
  int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    ragen_lineitem_row r = ragen_lineitem_at(&k, row0 + (uint64_t)i);
    if (shipdate) shipdate[i] = r.shipdate;
    if (rf) rf[i] = r.returnflag;
    if (ls) ls[i] = r.linestatus;
    if (qty) qty[i] = r.quantity;
    if (ep) ep[i] = r.extendedprice;
    if (disc) disc[i] = r.discount;
    if (tax) tax[i] = r.tax;
  }
}

int grid_for(int64_t n) {
  int64_t g = (n + 255) / 256;
  if (g > 148 * 32) g = 148 * 32;
  return g < 1 ? 1 : (int)g;
}

}  // namespace

// Returns 0 on success, else the cudaError_t value.
RAGEN_API int ragen_int32_dev(uint64_t seed, uint64_t row0, int64_t n, int32_t* d_x, void* stream) {
  if (n <= 0) return 0;
  k_int32<<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(ragen_key(seed, RAGEN_S_INT32), row0, n, d_x);
  return (int)cudaGetLastError();
}

RAGEN_API int ragen_lineitem_dev(uint64_t seed, uint32_t n_parts, uint64_t row0, int64_t n,
                                 int32_t* shipdate, uint8_t* returnflag, uint8_t* linestatus,
                                 int64_t* quantity, int64_t* extendedprice, int64_t* discount,
                                 int64_t* tax, void* stream) {
  if (n <= 0) return 0;
  k_lineitem<<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(
      ragen_lineitem_make_keys(seed, n_parts), row0, n, shipdate, returnflag, linestatus, quantity,
      extendedprice, discount, tax);
  return (int)cudaGetLastError();
}
