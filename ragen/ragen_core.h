/* ragen_core.h — seeded, counter-based synthetic input generator.
 *
 * INPUT GENERATION ONLY.  This module is shared by the CPU oracle's tests and
 * by the CUDA path's tests/bench; it holds none of the method's arithmetic
 * (no predicate, compaction, projection or aggregation).  Every value is a
 * pure function of (seed, stream, row index), so any row range — a shard, a
 * fission chunk, a test slice — is generated independently and identically
 * on the host (ragen.cu, host threads) and on the device (ragen.cu kernels).
 *
 * Recipes:
 *  - int32 column: "random 32-bit integers representing compressed row data"
 *    (§II/§III-B): uniform over all 2^32 bit
 *    patterns.
 *  - lineitem SoA: the seven Q1 columns (§V) drawn per row
 *    with the TPC-H §4.2.3 rules restated in SURVEY C15 (no orders table).
 */
#ifndef RAGEN_CORE_H
#define RAGEN_CORE_H

#include <stdint.h>

#if defined(__CUDACC__)
#define RAGEN_HD __host__ __device__ __forceinline__
#else
#define RAGEN_HD static inline
#endif

/* stream ids: one independent counter stream per drawn quantity */
enum {
  RAGEN_S_INT32 = 0,
  RAGEN_S_ORDERDATE = 1,
  RAGEN_S_SHIPOFF = 2,
  RAGEN_S_RECEIPTOFF = 3,
  RAGEN_S_RFCOIN = 4,
  RAGEN_S_QTY = 5,
  RAGEN_S_DISC = 6,
  RAGEN_S_TAX = 7,
  RAGEN_S_PARTKEY = 8
};

/* TPC-H calendar (days since 1970-01-01) */
#define RAGEN_STARTDATE 8035   /* 1992-01-01 */
#define RAGEN_LAST_ORDERDATE 10440 /* 1998-08-02 = ENDDATE - 151 */
#define RAGEN_CURRENTDATE 9298 /* 1995-06-17 */

RAGEN_HD uint64_t ragen_mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* per-(seed, stream) key; draw i of that stream = mix(key + i) */
RAGEN_HD uint64_t ragen_key(uint64_t seed, uint32_t stream) {
  return ragen_mix64(seed ^ ((uint64_t)stream << 56));
}

RAGEN_HD uint64_t ragen_draw(uint64_t key, uint64_t i) { return ragen_mix64(key + i); }

/* uniform integer in [lo, lo + span) from the high 32 bits (multiply-shift) */
RAGEN_HD int64_t ragen_uniform(uint64_t h, int64_t lo, uint32_t span) {
  return lo + (int64_t)(((h >> 32) * (uint64_t)span) >> 32);
}

RAGEN_HD int32_t ragen_int32_at(uint64_t key_int32, uint64_t i) {
  return (int32_t)(uint32_t)(ragen_draw(key_int32, i) >> 32);
}

typedef struct {
  uint64_t k_orderdate, k_shipoff, k_receiptoff, k_rfcoin, k_qty, k_disc, k_tax, k_partkey;
  uint32_t n_parts; /* partkey ~ U[1, n_parts], n_parts = 200000*SF */
} ragen_lineitem_keys;

RAGEN_HD ragen_lineitem_keys ragen_lineitem_make_keys(uint64_t seed, uint32_t n_parts) {
  ragen_lineitem_keys k;
  k.k_orderdate = ragen_key(seed, RAGEN_S_ORDERDATE);
  k.k_shipoff = ragen_key(seed, RAGEN_S_SHIPOFF);
  k.k_receiptoff = ragen_key(seed, RAGEN_S_RECEIPTOFF);
  k.k_rfcoin = ragen_key(seed, RAGEN_S_RFCOIN);
  k.k_qty = ragen_key(seed, RAGEN_S_QTY);
  k.k_disc = ragen_key(seed, RAGEN_S_DISC);
  k.k_tax = ragen_key(seed, RAGEN_S_TAX);
  k.k_partkey = ragen_key(seed, RAGEN_S_PARTKEY);
  k.n_parts = n_parts ? n_parts : 1u;
  return k;
}

typedef struct {
  int32_t shipdate;
  uint8_t returnflag, linestatus;
  int64_t quantity, extendedprice, discount, tax; /* x100 fixed point */
} ragen_lineitem_row;

/* One lineitem row (TPC-H §4.2.3 as restated in SURVEY C15). */
RAGEN_HD ragen_lineitem_row ragen_lineitem_at(const ragen_lineitem_keys* k, uint64_t i) {
  ragen_lineitem_row r;
  int32_t orderdate = (int32_t)ragen_uniform(ragen_draw(k->k_orderdate, i), RAGEN_STARTDATE,
                                             RAGEN_LAST_ORDERDATE - RAGEN_STARTDATE + 1);
  int32_t shipdate = orderdate + (int32_t)ragen_uniform(ragen_draw(k->k_shipoff, i), 1, 121);
  int32_t receiptdate = shipdate + (int32_t)ragen_uniform(ragen_draw(k->k_receiptoff, i), 1, 30);
  int64_t qty_units = ragen_uniform(ragen_draw(k->k_qty, i), 1, 50);
  int64_t pk = ragen_uniform(ragen_draw(k->k_partkey, i), 1, k->n_parts);
  int64_t retail_cents = 90000 + ((pk / 10) % 20001) + 100 * (pk % 1000);
  r.shipdate = shipdate;
  if (receiptdate <= RAGEN_CURRENTDATE)
    r.returnflag = (ragen_draw(k->k_rfcoin, i) >> 63) ? (uint8_t)'R' : (uint8_t)'A';
  else
    r.returnflag = (uint8_t)'N';
  r.linestatus = (shipdate > RAGEN_CURRENTDATE) ? (uint8_t)'O' : (uint8_t)'F';
  r.quantity = qty_units * 100;
  r.extendedprice = qty_units * retail_cents;
  r.discount = ragen_uniform(ragen_draw(k->k_disc, i), 0, 11);
  r.tax = ragen_uniform(ragen_draw(k->k_tax, i), 0, 9);
  return r;
}

#endif /* RAGEN_CORE_H */
