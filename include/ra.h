/* ra.h — C ABI of libra.so: the fused relational-operator hot path of
 * Wu, Diamos, Wang, Cadambi, Yalamanchili, Chakradhar, "Optimizing Data
 * Warehousing Applications for GPUs Using Kernel Fusion/Fission" (IPDPSW 2012),
 * built B200-native (sm_100a).
 *
 * Citations are PAPER.md line numbers with the section/figure/table they sit
 * in; "SURVEY Cn" = the reading of the paper recorded in SURVEY.md §8(c) and
 * DESIGN.md; EXT:TPC-H = the TPC-H specification (paper ref [9], L1791-1792).
 *
 * Conventions for every entry point
 *  - Plain pointers and sizes only.  "d_" = device pointer, "h_" = host pointer.
 *    All buffers are caller-owned; the library never allocates device memory.
 *  - Stream-ordered entry points (ra_select, ra_select_chain, ra_q1) enqueue
 *    work on `stream` and return immediately; results are valid once the
 *    caller synchronises that stream.  ra_fission_run and ra_q1_finalize are
 *    synchronous.
 *  - Return value: RA_OK or a negative RA_E_* code; nothing is enqueued when
 *    an argument check fails.  ra_last_error() gives a thread-local message.
 *    No exception or abort crosses the ABI.
 *  - Calls are reentrant given distinct workspaces; a workspace may be reused
 *    by successive calls ordered on one stream.
 *  - Workspaces must be zero-filled once after allocation (ra_workspace_init
 *    or any memset); the library keeps them self-cleaning afterwards for any
 *    number of calls of the SAME entry point with any n the size allows
 *    (select status words carry a launch-epoch tag; the launch before the tag
 *    wraps clears every status word the workspace has carried; data other
 *    than status words lives at the 256-B aligned end of the workspace).
 *    A workspace handed to a DIFFERENT entry point must be re-initialised
 *    first: another layout's data could read as a status word.
 *  - ws_bytes may exceed the required size by any amount.
 */
#ifndef RA_H
#define RA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Same type as cudaStream_t / CUstream; NULL = the legacy default stream. */
typedef struct CUstream_st* ra_stream_t;

/* ------------------------------------------------------------ error codes */
#define RA_OK 0
#define RA_E_INVAL (-1)       /* null pointer with n > 0, bad op, k > RA_MAX_PREDS,
                                 k < 0, n < 0, chunk_rows <= 0, misaligned pointer,
                                 n >= 2^32 where a call bounds n */
#define RA_E_CAPACITY (-2)    /* (synchronous calls) result larger than out_cap:
                                 the first out_cap values are written and the
                                 count output holds the full (required) count */
#define RA_E_DOMAIN (-3)      /* ra_q1_finalize: a partial reported rows outside
                                 the Q1 domain (see ra_q1_partial.status) */
#define RA_E_NOT_PINNED (-4)  /* ra_fission_run: a host buffer is not page-locked */
#define RA_E_CUDA (-5)        /* a CUDA runtime call failed (message has details) */
#define RA_E_WORKSPACE (-6)   /* ws_bytes smaller than the *_workspace_bytes size */

/* Thread-local message describing the last non-RA_OK return on this thread. */
const char* ra_last_error(void);

/* ABI version (bumped on any layout change). */
int ra_version(void);

/* Number of CUDA kernels this process has launched through libra.so
 * (monotonic; used by bench.py to report gpu_launches). */
uint64_t ra_kernel_launches(void);

/* Zero-fill a workspace (cudaMemsetAsync).  Needed once after allocation. */
int ra_workspace_init(void* d_ws, size_t ws_bytes, ra_stream_t stream);

/* ================================================================ SELECT
 * Predicate: the element compared with a constant, signed int32 —
 * "d < THRESHOLD" (Table III, §III-A) and "field.0==2" (Table I,
 * L153-156); SURVEY C1.  A chain is the conjunction of its predicates
 * (back-to-back SELECTs, Fig 2(a)).
 */
#define RA_MAX_PREDS 8
enum { RA_LT = 0, RA_LE = 1, RA_GT = 2, RA_GE = 3, RA_EQ = 4, RA_NE = 5 };

typedef struct {
  int32_t op;    /* RA_LT .. RA_NE */
  int32_t value; /* the constant */
} ra_pred;

/* Device workspace needed by ra_select / ra_select_chain for n rows.
 * fused != 0: one pass (tile status words only, ~2*8*n/4096 B + 256 B).
 * fused == 0: the unfused composition also keeps two intermediate int32[n]
 * relations on the device ("without round trip", L972-984). */
size_t ra_select_workspace_bytes(int64_t n, int k, int fused);

/* Single SELECT: d_out[0..count) = the elements of d_in[0..n) satisfying
 * `pred`, in input order; *d_count = count (int64, device).
 *
 * The paper's four stages — partition, filter, buffer, gather (Fig 3,
 * L303-310, L479-485) — run as ONE kernel: each CTA takes an 8192-row tile by
 * atomic ticket (partition), evaluates the predicate in registers (filter),
 * compacts matches in shared memory via warp ballots/scans (buffer) and
 * obtains its global output offset by a decoupled look-back over the tile
 * status words instead of the paper's global sync + second gather kernel
 * (gather).  Output order is the input order.
 *
 *  d_in      int32[n], 4-byte aligned (any sub-view of a device buffer)
 *  n         >= 0; n = 0 writes *d_count = 0
 *  d_out     int32[out_cap], 4-byte aligned; if count > out_cap only the first
 *            out_cap values are written, *d_count still holds the full count
 *  d_count   int64, device
 *  d_ws      workspace of ra_select_workspace_bytes(n, 1, 1) bytes (zeroed once)
 */
int ra_select(const int32_t* d_in, int64_t n, ra_pred pred, int32_t* d_out, int64_t out_cap,
              int64_t* d_count, void* d_ws, size_t ws_bytes, ra_stream_t stream);

/* Chain of k back-to-back SELECTs over one input (Fig 2(a), Fig 6).
 *  h_preds   host array of k predicates, 0 <= k <= RA_MAX_PREDS; k = 0 copies
 *  fused     != 0: one kernel evaluates all k predicates per element in
 *            registers — one partition/buffer/gather for the chain (L784-785,
 *            L812-814); the conjunction is simplified once on the host to an
 *            interval plus != exclusions (the Table III compiler benefit,
 *            L790-805).
 *            == 0: the unfused composition — k single-predicate passes with
 *            device-resident intermediates in d_ws (the paper's "without
 *            round trip" baseline, L972-984).  Same output (L580-581).
 * Other arguments as ra_select; ws sized by ra_select_workspace_bytes(n, k, fused).
 */
int ra_select_chain(const int32_t* d_in, int64_t n, const ra_pred* h_preds, int k, int fused,
                    int32_t* d_out, int64_t out_cap, int64_t* d_count, void* d_ws,
                    size_t ws_bytes, ra_stream_t stream);

/* Multi-GPU SELECT exchange, device side: rank r
 * selected from its own contiguous row range; after an all_gather of the
 * per-rank counts (NCCL, by the caller) its output belongs at the sum of the
 * counts of ranks < r — the gather stage's "correct position in the final
 * array" (Fig 3) one level up.  One small kernel, stream-ordered.
 *
 *  d_counts   device int64[n_ranks], 1 <= n_ranks <= RA_MAX_RANKS, the counts
 *             in rank order
 *  d_offsets  device int64[n_ranks] or NULL: exclusive prefix sums
 *  d_total    device int64 or NULL: the sum (not both NULL)
 *  All pointers 8-byte aligned. */
#define RA_MAX_RANKS 65536

int ra_select_offsets(const int64_t* d_counts, int n_ranks, int64_t* d_offsets, int64_t* d_total,
                      ra_stream_t stream);

/* ============================================================ TPC-H Q1
 * SELECT (l_shipdate <= cutoff) -> PROJECT (disc_price = price*(1-disc),
 * charge = disc_price*(1+tax)) -> GROUP BY (returnflag, linestatus)
 * SUM/COUNT, in one kernel with private accumulators and no HBM
 * intermediates (Fig 2(g)(h); Q1 plan §V; EXT:TPC-H;
 * SURVEY C8-C13).  The plan's JOINs are identities in a positional column
 * store and its SORT orders at most 6 groups (C9): neither is executed.
 *
 * Columns (SoA, device, n rows each; decimals are int64 fixed point x100, C10):
 *  shipdate int32 days since 1970-01-01; returnflag/linestatus bytes;
 *  quantity, extendedprice, discount, tax int64 x100.
 * Domain (checked on the SELECTED rows; violations are reported through
 * ra_q1_partial.status and such rows are not accumulated):
 *  returnflag in {'A','N','R'}, linestatus in {'F','O'}        (status bit 0)
 *  0 <= quantity, extendedprice < 2^31; 0 <= discount, tax <= 100 (status bit 1)
 * n < 2^32 per call.  Pointers must be naturally aligned.
 */
#define RA_Q1_GROUPS 6 /* slot = 2*rf + ls, rf: A=0 N=1 R=2, ls: F=0 O=1 */

typedef struct {
  const int32_t* shipdate;
  const uint8_t* returnflag;
  const uint8_t* linestatus;
  const int64_t* quantity;
  const int64_t* extendedprice;
  const int64_t* discount;
  const int64_t* tax;
} ra_lineitem;

/* Exact per-group sums.  Scales: qty/price/disc x1e2, disc_price x1e4,
 * charge x1e6; disc_price and charge are 128-bit (lo + hi<<64), C11. */
typedef struct {
  int64_t count;
  int64_t sum_qty;
  int64_t sum_base_price;
  int64_t sum_disc;
  uint64_t sum_disc_price_lo;
  int64_t sum_disc_price_hi;
  uint64_t sum_charge_lo;
  int64_t sum_charge_hi;
} ra_q1_group;

/* One shard's partial aggregate; shards combine by exact slotwise addition. */
typedef struct {
  uint32_t status;   /* OR of domain bits over selected rows (0 = clean) */
  uint32_t n_groups; /* RA_Q1_GROUPS */
  uint64_t rows;     /* rows scanned */
  ra_q1_group group[RA_Q1_GROUPS];
} ra_q1_partial;

/* One output row of Q1 (ORDER BY returnflag, linestatus). */
typedef struct {
  uint8_t returnflag, linestatus, _pad[6];
  int64_t count_order;
  int64_t sum_qty;        /* x1e2 */
  int64_t sum_base_price; /* x1e2 */
  int64_t sum_disc;       /* x1e2 */
  uint64_t sum_disc_price_lo; /* x1e4, 128-bit */
  int64_t sum_disc_price_hi;
  uint64_t sum_charge_lo;     /* x1e6, 128-bit */
  int64_t sum_charge_hi;
  double avg_qty, avg_price, avg_disc; /* (double)sum / (double)(100*count), C12 */
} ra_q1_row;

size_t ra_q1_workspace_bytes(int64_t n);

/* Enqueue the fused Q1 kernel.  h_cols: host struct of DEVICE column
 * pointers; shipdate_cutoff inclusive (TPC-H DELTA=90: 10471 = 1998-09-02);
 * d_partial: device ra_q1_partial written completely (all 6 slots). */
int ra_q1(const ra_lineitem* h_cols, int64_t n, int32_t shipdate_cutoff,
          ra_q1_partial* d_partial, void* d_ws, size_t ws_bytes, ra_stream_t stream);

/* Host: sum n_partials partials exactly (row-range shards, fission chunks),
 * drop empty groups, order by (returnflag, linestatus), compute the AVGs
 * ("Aggregate/Unique", Fig 17(a)).  h_rows holds >= 6 rows.
 * Returns RA_E_DOMAIN (rows still filled) if any partial has status != 0. */
int ra_q1_finalize(const ra_q1_partial* h_partials, int n_partials, ra_q1_row* h_rows,
                   int* n_rows);

/* ============================================================ SEVERAL SELECTs
 * Several SELECT operators filtering the same input (Fig 2(c)
 * L286-288, "different SELECT operators need to filter the same input data").
 * One fused pass reads the input once, evaluates every output's predicate
 * chain in registers and compacts each output separately (order-preserving;
 * the M tile aggregates travel in ceil(M/2) look-back status words).  Output
 * o equals ra_select_chain(d_in, chains[o]).  Stream-ordered.
 *
 *  d_in          device int32[n] (4-B aligned), n < 2^34
 *  h_chains[o]   host array of ks[o] predicates (0 <= ks[o] <= RA_MAX_PREDS)
 *  M             number of outputs, 1 <= M <= RA_MAX_OUTPUTS
 *  d_outs[o]     device int32[out_caps[o]] (4-B aligned; may be NULL if
 *                out_caps[o] == 0)
 *  d_counts[o]   device int64 (8-B aligned): output o's size (the required size)
 *  d_ws          ra_select_multi_workspace_bytes(n) bytes, 256-B aligned,
 *                zeroed once (tile status words only)
 * Rows beyond out_caps[o] are not written (the count is still exact).
 * RA_E_INVAL on a bad argument, RA_E_WORKSPACE if ws_bytes is too small. */
#define RA_MAX_OUTPUTS 4

size_t ra_select_multi_workspace_bytes(int64_t n);

int ra_select_multi(const int32_t* d_in, int64_t n, const ra_pred* const* h_chains, const int* ks, int M,
                    int32_t* const* d_outs, const int64_t* out_caps, int64_t* const* d_counts, void* d_ws,
                    size_t ws_bytes, ra_stream_t stream);

/* ============================================================ TUPLE SELECT
 * SELECT over a multi-column relation.  Table I's example
 * "select [field.0==2] x -> (2,False,b)" (L153-156) returns whole tuples; in a
 * column store field 0 is the int32 key column and the other fields are
 * payload columns.  One fused pass evaluates the predicate chain on the key
 * and compacts the selected rows' ids (order-preserving, single pass with
 * decoupled look-back), also leaving per-tile order masks in the workspace;
 * the payload fields are then placed on the same stream (the paper's stage 4
 * "gather", Fig 3) by one of two kernels, chosen on the device from
 * the count: few selected rows -> a gather at the ids; many -> a streaming
 * compaction that reads each payload column once, in order.  Both give the
 * same result (environment RA_TUPLE_GATHER=1 forces the gather: diagnostics).
 * With k = 0 every row is kept: PROJECT (Table I) of the payload
 * fields.  Output = the selected tuples, stream-ordered.
 *
 *  d_key        device int32[n] (4-B aligned), n < 2^32
 *  h_preds, k   as ra_select_chain (host array, k <= RA_MAX_PREDS)
 *  d_rowids     device uint32[out_cap] or NULL: selected row ids (0-based)
 *  h_payloads   host array of m <= RA_MAX_PAYLOAD fields {col, out,
 *               elem_bytes}: col device [n] elements of elem_bytes (4 or 8,
 *               naturally aligned), out device [out_cap] elements; may be
 *               NULL when m == 0
 *  d_count      device int64: number selected (the required size)
 *  d_ws         ra_select_rows_workspace_bytes(n, k) bytes, zeroed once
 * Rows beyond out_cap are not written (count is still exact). */
#define RA_MAX_PAYLOAD 4

typedef struct {
  const void* col;
  void* out;
  int32_t elem_bytes;
  int32_t _pad;
} ra_payload;

size_t ra_select_rows_workspace_bytes(int64_t n, int k);

int ra_select_rows(const int32_t* d_key, int64_t n, const ra_pred* h_preds, int k, uint32_t* d_rowids,
                   const ra_payload* h_payloads, int m, int64_t out_cap, int64_t* d_count, void* d_ws,
                   size_t ws_bytes, ra_stream_t stream);

/* ============================================================= FISSION
 * Host-resident SELECT chain with kernel fission (§IV; pipelined
 * segments §IV-B; fusion+fission §IV-C).
 * The input is split into contiguous chunks of chunk_rows (last one shorter);
 * chunk c runs on streams[c % n_streams]: H2D copy -> select_chain kernel ->
 * D2H of exactly that chunk's count into h_out at the running offset (the
 * paper's "CPU gather", L1466-1468).  Copies of one chunk overlap the kernel
 * of another; time ~ max(H2D, compute, D2H) (L1504-1509).  Output equals
 * ra_select_chain on the whole input (C16).  Synchronous.
 *
 *  h_in            pinned host int32[n]
 *  h_preds, k      as ra_select_chain; fused selects the chain kernel form
 *  chunk_rows      > 0 (chunk_rows >= n with one stream = the "serial" mode)
 *  streams         n_streams >= 1 CUDA streams of the current device
 *  h_out           pinned host int32[out_cap]
 *  h_count         host int64: total selected (the required size if > out_cap)
 *  h_chunk_counts  pinned host int64[ceil(n/chunk_rows)]: per-chunk counts,
 *                  written by the device through its mapped alias
 *  d_ws            ra_fission_workspace_bytes(chunk_rows, n_streams, k, fused)
 * Returns RA_E_CAPACITY if the total exceeds out_cap (first out_cap written).
 */
size_t ra_fission_workspace_bytes(int64_t chunk_rows, int n_streams, int k, int fused);

int ra_fission_run(const int32_t* h_in, int64_t n, const ra_pred* h_preds, int k, int fused,
                   int64_t chunk_rows, const ra_stream_t* streams, int n_streams, int32_t* h_out,
                   int64_t out_cap, int64_t* h_count, int64_t* h_chunk_counts, void* d_ws,
                   size_t ws_bytes);

/* Host-resident TPC-H Q1 under kernel fission: the paper
 * applies fission to Q1's fused input stage (L1565-1566, L1669-1671).  The
 * seven columns are streamed in contiguous chunks of chunk_rows (last one
 * shorter); chunk c runs on streams[c % n_streams]: H2D of its 38 B/row ->
 * fused Q1 kernel accumulating into that stream's device partial.  Chunks of
 * one stream are ordered by the stream, so the host never waits inside the
 * loop; at the end the n_streams partials are summed exactly (the same
 * slotwise addition as row-range shards) into *h_partial.  Synchronous.
 *
 *  h_cols      host struct of PINNED host column pointers (layout and domain
 *              as ra_q1), n < 2^32 rows
 *  chunk_rows  > 0; chunk_rows >= n with one stream = the serial mode
 *  streams     n_streams >= 1 CUDA streams of the current device
 *  h_partial   host ra_q1_partial: the whole query's partial (pass it to
 *              ra_q1_finalize)
 *  d_ws        ra_q1_fission_workspace_bytes(chunk_rows, n_streams), 256-B
 *              aligned
 * Result identical to ra_q1 over the whole table (partition additivity). */
size_t ra_q1_fission_workspace_bytes(int64_t chunk_rows, int n_streams);

int ra_q1_fission_run(const ra_lineitem* h_cols, int64_t n, int32_t shipdate_cutoff,
                      int64_t chunk_rows, const ra_stream_t* streams, int n_streams,
                      ra_q1_partial* h_partial, void* d_ws, size_t ws_bytes);

/* ====================================================== NARROW Q1 (f4)
 * Compressed lineitem for Q1.  The paper's relations are
 * "compressed row data" (§III-D) and it names compression as the way
 * to cut transfer volume (§VI).  The seven Q1 columns (38 B/row)
 * are re-encoded losslessly into six narrow columns (11 B/row); Q1 over them
 * yields exactly the partial ra_q1 yields over the wide columns.
 *
 *   shipdate       uint16  days since 1970-01-01            (0 .. 65535)
 *   group          uint8   slot = 2*rf + ls (rf A=0 N=1 R=2,
 *                          ls F=0 O=1), i.e. RA_Q1 slot order (0 .. 5)
 *   quantity       uint16  x100                              (0 .. 65535)
 *   discount, tax  uint8   x100                              (0 .. 100)
 *   extendedprice  uint32  x100                              (0 .. 2^24-1)
 * Every TPC-H row fits (quantity <= 5000, price <= 10,495,000).
 * All column pointers are device pointers aligned to 16 bytes, n rows each. */
typedef struct {
  const uint16_t* shipdate;
  const uint8_t* group;
  const uint16_t* quantity;
  const uint8_t* discount;
  const uint8_t* tax;
  const uint32_t* extendedprice;
} ra_lineitem_narrow;

typedef struct {
  uint16_t* shipdate;
  uint8_t* group;
  uint16_t* quantity;
  uint8_t* discount;
  uint8_t* tax;
  uint32_t* extendedprice;
} ra_lineitem_narrow_out;

/* Encode n wide rows (h_cols: device columns, ra_q1 layout) into the narrow
 * columns h_out (device, 16-B aligned).  *d_status (device uint32) is
 * overwritten with the OR over ALL rows of: 1 = a flag byte outside
 * {A,N,R}x{F,O} (row encoded with group 0xFF), 2 = quantity, price, discount
 * or tax outside the narrow ranges (row encoded with group 0xFE),
 * 4 = shipdate outside 0..65535 (clamped).  A table with status 0 is an exact
 * re-encoding.  Stream-ordered; n < 2^32. */
int ra_q1_encode(const ra_lineitem* h_cols, int64_t n, const ra_lineitem_narrow_out* h_out,
                 uint32_t* d_status, ra_stream_t stream);

/* Fused Q1 over narrow columns: same workspace (ra_q1_workspace_bytes), same
 * cutoff convention and same output (ra_q1_partial, all 6 slots) as ra_q1.
 * A SELECTED row with group > 5 sets status bit 0, one with discount or tax
 * > 100 or price >= 2^24 sets status bit 1; such rows are not accumulated.
 * Stream-ordered; n < 2^32; columns 16-B aligned. */
int ra_q1_narrow(const ra_lineitem_narrow* h_cols, int64_t n, int32_t shipdate_cutoff,
                 ra_q1_partial* d_partial, void* d_ws, size_t ws_bytes, ra_stream_t stream);

/* Host-resident narrow Q1 under kernel fission (f1 x f4): as
 * ra_q1_fission_run, but h_cols holds PINNED host narrow columns (11 B/row
 * over PCIe instead of 38).  Result identical to ra_q1_narrow on the whole
 * table.  Synchronous.  d_ws: ra_q1_narrow_fission_workspace_bytes, 256-B
 * aligned. */
size_t ra_q1_narrow_fission_workspace_bytes(int64_t chunk_rows, int n_streams);

int ra_q1_narrow_fission_run(const ra_lineitem_narrow* h_cols, int64_t n, int32_t shipdate_cutoff,
                             int64_t chunk_rows, const ra_stream_t* streams, int n_streams,
                             ra_q1_partial* h_partial, void* d_ws, size_t ws_bytes);

#ifdef __cplusplus
}
#endif

#endif /* RA_H */
