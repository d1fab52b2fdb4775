/* oracle.c — plain, slow, obviously-correct CPU oracle of the hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_ipps_wudwcyc12_b200/ and include/), and imports nothing from it.
 * Single-threaded scalar C; every function follows the definition it cites,
 * with no blocking, fusion or reordering.
 *
 * Citations: PAPER.md line numbers (section / figure / table).  EXT:TPC-H =
 * the TPC-H specification the paper cites as ref [9];
 * its Q1 text is restated in SURVEY.md §8(c) C8.
 *
 * Pins (what fixes this code to something other than itself): see
 * tests/test_oracle_select.py and tests/test_oracle_q1.py — brute force on tiny
 * inputs, numpy boolean indexing, the Table I SELECT example, pyarrow
 * decimal128 and sqlite3 group-by, a hand-computed Q1 fixture
 * (tests/golden/q1_worked_example.txt), closed-form invariants.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_API __attribute__((visibility("default")))

/* Predicate: "d < THRESHOLD" (Table III, §III-A) and
 * "field.0 == 2" (Table I).  Signed int32 comparisons of the
 * element against a constant.  Op codes are this file's own. */
enum { ORACLE_LT = 0, ORACLE_LE = 1, ORACLE_GT = 2, ORACLE_GE = 3, ORACLE_EQ = 4, ORACLE_NE = 5 };

typedef struct {
  int32_t op;
  int32_t value;
} oracle_pred;

/* 1 if x satisfies (op, v), 0 if not, -1 for an unknown op. */
ORACLE_API int oracle_cmp(int32_t op, int32_t x, int32_t v) {
  switch (op) {
    case ORACLE_LT: return x < v;
    case ORACLE_LE: return x <= v;
    case ORACLE_GT: return x > v;
    case ORACLE_GE: return x >= v;
    case ORACLE_EQ: return x == v;
    case ORACLE_NE: return x != v;
    default: return -1;
  }
}

/* SELECT of a chain of k predicates (Table I; back-to-back SELECTs,
 * Fig 2(a); fused chain = second filter stage inserted after the
 * first, Fig 6 / L581-584): keep x[i] iff every predicate holds, preserving
 * input order (the gather puts matches at "their correct position in the
 * final array", L481-483).  k = 0 keeps everything.  out may be NULL (count
 * only).  Returns the number kept, or -1 for an invalid predicate. */
ORACLE_API int64_t oracle_select(const int32_t* x, int64_t n, const oracle_pred* P, int k,
                                 int32_t* out) {
  int64_t count = 0;
  for (int j = 0; j < k; ++j)
    if (oracle_cmp(P[j].op, 0, P[j].value) < 0) return -1;
  for (int64_t i = 0; i < n; ++i) {
    int keep = 1;
    for (int j = 0; j < k; ++j)
      if (!oracle_cmp(P[j].op, x[i], P[j].value)) keep = 0;
    if (keep) {
      if (out) out[count] = x[i];
      count++;
    }
  }
  return count;
}

/* Unfused composition sel(...sel(sel(x,[P0]),[P1])...,[Pk-1]): one SELECT per
 * predicate with a materialised intermediate ("without round trip", L972-984);
 * functionally equal to the fused chain (L580-581). */
ORACLE_API int64_t oracle_select_unfused(const int32_t* x, int64_t n, const oracle_pred* P, int k,
                                         int32_t* out) {
  if (k == 0) return oracle_select(x, n, P, 0, out);
  int32_t* a = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int32_t* b = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  if (!a || !b) {
    free(a);
    free(b);
    return -2;
  }
  int64_t m = n;
  memcpy(a, x, sizeof(int32_t) * (size_t)n);
  for (int j = 0; j < k; ++j) {
    m = oracle_select(a, m, &P[j], 1, b);
    if (m < 0) break;
    int32_t* t = a;
    a = b;
    b = t;
  }
  if (m > 0 && out) memcpy(out, a, sizeof(int32_t) * (size_t)m);
  free(a);
  free(b);
  return m;
}

/* Fission result: SELECT each contiguous chunk of `chunk` rows independently
 * (the last chunk shorter) and CPU-gather the chunk results in chunk order
 * (§IV-B, §IV-C "the CPU has to implement a gather stage",
 * L1466-1468). */
ORACLE_API int64_t oracle_select_chunked(const int32_t* x, int64_t n, const oracle_pred* P, int k,
                                         int64_t chunk, int32_t* out) {
  if (chunk <= 0) return -1;
  int64_t total = 0;
  for (int64_t c0 = 0; c0 < n; c0 += chunk) {
    int64_t len = (n - c0 < chunk) ? (n - c0) : chunk;
    int64_t m = oracle_select(x + c0, len, P, k, out ? out + total : NULL);
    if (m < 0) return m;
    total += m;
  }
  return total;
}

/* Several SELECTs filtering the same input (Fig 2(c): "different
 * SELECT operators need to filter the same input data"): output o is the
 * order-preserving SELECT of x by its own chain P[off[o] .. off[o]+k[o]),
 * exactly as oracle_select would give it; counts[o] receives its size.  One
 * pass over x (each element tested against every chain).  Returns 0, or -1
 * for an invalid predicate. */
ORACLE_API int oracle_select_multi(const int32_t* x, int64_t n, const oracle_pred* P, const int32_t* off,
                                   const int32_t* k, int M, int32_t* const* outs, int64_t* counts) {
  for (int o = 0; o < M; ++o) {
    counts[o] = 0;
    for (int j = 0; j < k[o]; ++j)
      if (oracle_cmp(P[off[o] + j].op, 0, P[off[o] + j].value) < 0) return -1;
  }
  for (int64_t i = 0; i < n; ++i) {
    for (int o = 0; o < M; ++o) {
      int keep = 1;
      for (int j = 0; j < k[o]; ++j)
        if (!oracle_cmp(P[off[o] + j].op, x[i], P[off[o] + j].value)) keep = 0;
      if (keep) {
        if (outs && outs[o]) outs[o][counts[o]] = x[i];
        counts[o]++;
      }
    }
  }
  return 0;
}

/* SELECT over a multi-column relation (Table I: "select
 * [field.0==2] x -> (2,False,b)" returns whole tuples; the first field is the
 * key).  Column store: `key` is field 0, cols[0..m) are further fields of
 * elem_bytes[j] bytes each (4 or 8).  A row is kept iff every predicate holds
 * on its key; kept rows come out in input order (L481-483) as their row index
 * (rowids, may be NULL) and as each field's value (outs[j], may be NULL).
 * With k = 0 every row is kept, which is PROJECT (Table I:
 * "project [0,2] x") when cols names the projected fields.  Returns the
 * number kept, -1 for an invalid predicate or element size. */
ORACLE_API int64_t oracle_select_rows(const int32_t* key, int64_t n, const oracle_pred* P, int k, int m,
                                      const void* const* cols, const int32_t* elem_bytes, int64_t* rowids,
                                      void* const* outs) {
  for (int j = 0; j < k; ++j)
    if (oracle_cmp(P[j].op, 0, P[j].value) < 0) return -1;
  for (int j = 0; j < m; ++j)
    if (elem_bytes[j] != 4 && elem_bytes[j] != 8) return -1;
  int64_t count = 0;
  for (int64_t i = 0; i < n; ++i) {
    int keep = 1;
    for (int j = 0; j < k; ++j)
      if (!oracle_cmp(P[j].op, key[i], P[j].value)) keep = 0;
    if (!keep) continue;
    if (rowids) rowids[count] = i;
    for (int j = 0; j < m; ++j)
      if (outs && outs[j])
        memcpy((char*)outs[j] + count * elem_bytes[j], (const char*)cols[j] + i * elem_bytes[j],
               (size_t)elem_bytes[j]);
    count++;
  }
  return count;
}

/* ------------------------------------------------------------------ Q1
 * TPC-H Q1 (EXT:TPC-H, restated SURVEY C8; the paper's plan Fig 17(a),
 * §V: SELECT on shipdate, JOINs assembling seven columns, SORT by
 * (returnflag, linestatus), arithmetic + aggregate/unique):
 *
 *   select l_returnflag, l_linestatus,
 *          sum(l_quantity), sum(l_extendedprice),
 *          sum(l_extendedprice*(1-l_discount)),
 *          sum(l_extendedprice*(1-l_discount)*(1+l_tax)),
 *          avg(l_quantity), avg(l_extendedprice), avg(l_discount), count(*)
 *   from lineitem where l_shipdate <= date '1998-12-01' - interval '90' day
 *   group by l_returnflag, l_linestatus order by l_returnflag, l_linestatus
 *
 * Decimals are int64 fixed point x100: the products carry
 * scales 1e4 (disc_price) and 1e6 (charge) with no intermediate rounding.
 * Sums are exact 128-bit integers.  The group key is the raw byte pair, so
 * any bytes are accepted (C13); groups with count 0 are omitted and the rows
 * come out ordered by (returnflag, linestatus) ascending.
 * AVG = (double)sum / (double)(100 * count): one IEEE division of exact
 * operands while both are < 2^53 (C12).
 *
 * status (the C-ABI's documented domain, include/ra.h, evaluated over the
 * SELECTED rows only):
 *   bit 0 — (returnflag, linestatus) outside {A,N,R} x {F,O}
 *   bit 1 — quantity or extendedprice outside [0, 2^31), or discount or tax
 *           outside [0, 100]
 */
typedef struct {
  uint8_t returnflag, linestatus, _pad[6];
  int64_t count_order;
  uint64_t sum_qty_lo;
  int64_t sum_qty_hi;
  uint64_t sum_base_price_lo;
  int64_t sum_base_price_hi;
  uint64_t sum_disc_price_lo;
  int64_t sum_disc_price_hi;
  uint64_t sum_charge_lo;
  int64_t sum_charge_hi;
  uint64_t sum_disc_lo;
  int64_t sum_disc_hi;
  double avg_qty, avg_price, avg_disc;
} oracle_q1_row;

typedef struct {
  int64_t cnt;
  __int128 sq, sp, sdp, sch, sd;
} oracle_q1_acc;

static void put128(__int128 v, uint64_t* lo, int64_t* hi) {
  *lo = (uint64_t)v;
  *hi = (int64_t)(v >> 64);
}

/* rows must hold up to 65536 entries; returns the number of groups. */
ORACLE_API int oracle_q1(const int32_t* shipdate, const uint8_t* returnflag,
                         const uint8_t* linestatus, const int64_t* quantity,
                         const int64_t* extendedprice, const int64_t* discount, const int64_t* tax,
                         int64_t n, int32_t cutoff, oracle_q1_row* rows, uint32_t* status) {
  oracle_q1_acc* acc = (oracle_q1_acc*)calloc(65536, sizeof(oracle_q1_acc));
  if (!acc) return -2;
  uint32_t st = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (!(shipdate[i] <= cutoff)) continue; /* WHERE l_shipdate <= cutoff */
    uint8_t rf = returnflag[i], ls = linestatus[i];
    int64_t q = quantity[i], p = extendedprice[i], d = discount[i], t = tax[i];
    int rf_ok = (rf == 'A' || rf == 'N' || rf == 'R');
    int ls_ok = (ls == 'F' || ls == 'O');
    if (!(rf_ok && ls_ok)) st |= 1u;
    if (q < 0 || q >= ((int64_t)1 << 31) || p < 0 || p >= ((int64_t)1 << 31) || d < 0 ||
        d > 100 || t < 0 || t > 100)
      st |= 2u;
    oracle_q1_acc* a = &acc[(int)rf * 256 + (int)ls]; /* GROUP BY */
    __int128 disc_price = (__int128)p * (100 - d);   /* l_extendedprice*(1-l_discount) */
    __int128 charge = disc_price * (100 + t);         /* ... *(1+l_tax) */
    a->cnt += 1;
    a->sq += q;
    a->sp += p;
    a->sdp += disc_price;
    a->sch += charge;
    a->sd += d;
  }
  int m = 0;
  for (int g = 0; g < 65536; ++g) { /* ORDER BY returnflag, linestatus */
    oracle_q1_acc* a = &acc[g];
    if (a->cnt == 0) continue;
    oracle_q1_row* r = &rows[m++];
    memset(r, 0, sizeof(*r));
    r->returnflag = (uint8_t)(g >> 8);
    r->linestatus = (uint8_t)(g & 255);
    r->count_order = a->cnt;
    put128(a->sq, &r->sum_qty_lo, &r->sum_qty_hi);
    put128(a->sp, &r->sum_base_price_lo, &r->sum_base_price_hi);
    put128(a->sdp, &r->sum_disc_price_lo, &r->sum_disc_price_hi);
    put128(a->sch, &r->sum_charge_lo, &r->sum_charge_hi);
    put128(a->sd, &r->sum_disc_lo, &r->sum_disc_hi);
    double den = (double)(a->cnt * 100);
    r->avg_qty = (double)a->sq / den;
    r->avg_price = (double)a->sp / den;
    r->avg_disc = (double)a->sd / den;
  }
  free(acc);
  if (status) *status = st;
  return m;
}

ORACLE_API int oracle_q1_row_size(void) { return (int)sizeof(oracle_q1_row); }
