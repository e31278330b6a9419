/*
 * ltpg.h -- C-ABI of the B200-native LTPG per-batch pipeline.
 *
 * One call of ltpg_run_batch() runs one batch of LTPG's deterministic
 * optimistic concurrency control (§IV, Alg. 1):
 *   execute (readMem / recordTID / recordLS)
 *   -> conflict detection (rcheck / wcheck)
 *   -> write-back (getStatus -> writeMem / Abort)
 * with TID order as the serial order and conflicting txns
 * returned for re-execution in the next batch with their original TIDs
 * (P:110-112).  Commit rule (R1): txn of rank r aborts
 * iff it reads or writes a conflict unit that a smaller rank wrote (RAW/WAW),
 * or adds to a unit a smaller rank plainly wrote; delayed ADDs commute.
 * A conflict unit is (table, row, column group) (P:239 row-level splitting).
 *
 * Conventions (all functions):
 *  - Every call returns int: 0 = LTPG_OK, negative = error; no C++ exception
 *    crosses the ABI.  ltpg_last_error() gives a one-line reason.
 *  - The caller owns every input and result buffer; the library owns the
 *    device store, indexes, conflict marks and scratch (plain cudaMalloc).
 *  - Pointers are HOST pointers unless the corresponding *_on_device flag is
 *    set, in which case they are device pointers on the db's device (e.g. a
 *    torch tensor's data_ptr()).  Host pointers should be pinned for speed.
 *  - Validation happens before any mutation: a malformed batch returns
 *    LTPG_EINVAL and leaves the database unchanged (batch-level atomicity).
 *    LTPG_ECAPACITY (append region full) is also detected before write-back.
 *    A CUDA fault poisons the db: later calls return LTPG_EPOISONED.
 *  - All integer state: int64 columns with wrap-around (uint64) arithmetic,
 *    u64 keys (0xFFFFFFFFFFFFFFFF reserved), u32 batch ranks as conflict TIDs.
 */
#ifndef LTPG_H
#define LTPG_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define LTPG_API __attribute__((visibility("default")))
#else
#define LTPG_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ---------------------------------------------------------- */
enum {
  LTPG_OK = 0,
  LTPG_EINVAL = -1,     /* malformed argument or batch; nothing changed            */
  LTPG_ENOMEM = -2,     /* device allocation failed                                */
  LTPG_ECAPACITY = -3,  /* an append region / index would overflow; nothing changed */
  LTPG_ECUDA = -4,      /* CUDA runtime error (db poisoned)                         */
  LTPG_ERESERVED5 = -5, /* (unused)                                                 */
  LTPG_EPOISONED = -6,  /* an earlier device error poisoned this db: destroy it      */
  LTPG_EINTERNAL = -7   /* broken invariant (e.g. a required TPC-C row missing)      */
};

/* ---- OPS mode: one 16-byte record per operation ------------------------------ */
enum { LTPG_SELECT = 0, LTPG_UPDATE = 1, LTPG_ADD = 2, LTPG_INSERT = 3, LTPG_DELETE = 4, LTPG_SCAN = 5 };
#define LTPG_COL_COUNT 0xFFFFu      /* SCAN column: return the number of present keys */
#define LTPG_STATIC 0xFFu           /* col_group value: column never written, reads unmarked */
#define LTPG_NOT_FOUND INT64_MIN    /* read result for an absent key */

/* Operation semantics (DESIGN.md §"OPS semantics"):
 *  SELECT(t,key,col)       -> value of col in the pre-batch snapshot, or NOT_FOUND.
 *  UPDATE(t,key,col,arg)   read-modify-write col <- col + arg; returns the pre-image.
 *  ADD(t,key,col,arg)      delayed blind add on an ADD column; returns 0.
 *  INSERT(t,key,arg)       new row, column c = arg + c; returns 1, or 0 and a user
 *                          abort (status 2) if key is present in the snapshot.
 *  DELETE(t,key)           returns 1 (deleted) or NOT_FOUND.
 *  SCAN(t,key,col,aux=len) keys [key, key+len): sum of col over present keys
 *                          (or their count if col == LTPG_COL_COUNT).
 * Ops on absent keys return NOT_FOUND and count as a read of the key's row.
 * Within one txn a key that is written is touched by no other op (EINVAL). */
typedef struct {
  uint64_t key;
  uint8_t kind;
  uint8_t table;
  uint16_t col;
  uint32_t aux;
} ltpg_op;

/* ---- PROC mode: TPC-C stored procedures, 128-byte parameter blocks ---- */
enum { LTPG_NEW_ORDER = 0, LTPG_PAYMENT = 1, LTPG_ORDER_STATUS = 2, LTPG_DELIVERY = 3, LTPG_STOCK_LEVEL = 4 };
#define LTPG_PARAM_BYTES 128
#define LTPG_PROC_RESULTS 4         /* int64 result slots per PROC txn */

/* TPC-C schema (integer-only): table ids and column order.  Keys:
 *   W = w;  D = w*10+d;  C = D*3000+c;  I = i;  S = w*100000+i;
 *   O = NO = (D<<32)|o;  OL = O*16+ol;  HISTORY is keyless.            */
enum { LTPG_T_WAREHOUSE = 0, LTPG_T_DISTRICT = 1, LTPG_T_CUSTOMER = 2, LTPG_T_HISTORY = 3,
       LTPG_T_NEW_ORDER = 4, LTPG_T_ORDER = 5, LTPG_T_ORDER_LINE = 6, LTPG_T_ITEM = 7,
       LTPG_T_STOCK = 8, LTPG_TPCC_TABLES = 9 };
/* WAREHOUSE  : W_TAX, W_YTD
 * DISTRICT   : D_TAX, D_YTD, D_NEXT_O_ID, D_NEXT_DELIV_O_ID
 * CUSTOMER   : C_DISCOUNT, C_CREDIT, C_LAST, C_FIRST, C_INIT_O_ID, C_BALANCE,
 *              C_YTD_PAYMENT, C_PAYMENT_CNT, C_DELIVERY_CNT
 * HISTORY    : H_C_ID, H_C_D_ID, H_C_W_ID, H_D_ID, H_W_ID, H_DATE, H_AMOUNT, H_TID, H_SEQ
 * NEW_ORDER  : NO_O_ID
 * ORDER      : O_C_ID, O_ENTRY_D, O_OL_CNT, O_ALL_LOCAL, O_CARRIER_ID
 * ORDER_LINE : OL_I_ID, OL_SUPPLY_W_ID, OL_QUANTITY, OL_AMOUNT, OL_DELIVERY_D
 * ITEM       : I_PRICE, I_IM_ID
 * STOCK      : S_QUANTITY, S_YTD, S_ORDER_CNT, S_REMOTE_CNT
 * Column groups / ADD flags select "strict" or "delayed" mode. */

/* Parameter blocks (little endian, 128 bytes):
 * NewOrder   : u16 w | u8 d | u8 n_lines | u16 c | u8 rbk | u8 pad |
 *              15 x { u32 i | u16 supply_w | u8 qty | u8 pad }
 * Payment    : u16 w | u8 d | u8 by_name | u16 c_w | u8 c_d | u8 pad | u16 c_id |
 *              u16 c_last | u32 pad | i64 amount | ...
 * OrderStatus: u16 w | u8 d | u8 by_name | u16 c_id | u16 c_last | ...
 * Delivery   : u16 w | u8 carrier | ...
 * StockLevel : u16 w | u8 d | u8 threshold | ...
 * Results (4 x int64 per txn):
 * NewOrder [o_id (0 unless committed), total, sum(OL_AMOUNT), 0]
 * Payment  [c_id, C_BALANCE pre-image (strict) or 0 (delayed), 0, 0]
 * OrderStatus [c_id, C_BALANCE, O_CARRIER_ID, sum(OL_DELIVERY_D)]
 * Delivery [districts delivered, sum of delivered OL_AMOUNT, 0, 0]
 * StockLevel [low-stock count, D_NEXT_O_ID, 0, 0]                               */

/* ---- txn status ------------------------------------------------------------- */
enum { LTPG_ST_CONFLICT = 0, LTPG_ST_COMMIT = 1, LTPG_ST_USER_ABORT = 2 };

/* ---- configuration ------------------------------------------------------------ */
#define LTPG_FLAG_NO_GROUPING   (1u << 0)  /* A/B: disable adaptive warp division (§V-B) */
#define LTPG_FLAG_NO_MARK_FILTER (1u << 1) /* A/B: always issue the atomicMin mark        */
#define LTPG_FLAG_REORDER       (1u << 2)  /* NEXT-1 logical reordering: abort iff
                                              WAW or (RAW and WAR); keeps per-unit min reader marks */
#define LTPG_FLAG_UNFUSED       (1u << 3)  /* A/B: OPS mode runs validate+division and execute as
                                              two kernels with global per-kind lists          */
#define LTPG_FLAG_RESERVED_4    (1u << 4)  /* reserved (EINVAL); round 1's ncclAllReduce exchange
                                              baseline, removed: it could not run with several
                                              ranks on one GPU, the only multi-rank setup tested */
#define LTPG_FLAG_LARGE_BUCKETS (1u << 5)  /* NEXT-3: popularity is identified per batch
                                              ("in real time"): a table with E = T/D > 1
                                              (T = txns of the batch accessing it, D = its loaded
                                              rows) records that batch's marks in large-sized
                                              buckets of ceil(E/32)*32 sub-slots (TID mod s_u),
                                              folded per unit before detection.  Buckets are
                                              allocated at load for tables with max_txns/rows > 1
                                              (at most 64 MB each).  Result-identical          */
#define LTPG_FLAG_GRAPH         (1u << 6)  /* run each batch's device work as a captured CUDA graph,
                                              replayed for later batches of the same shape
                                              (see ltpg_run_batch); result-identical          */
#define LTPG_FLAG_L2_PERSIST_MARKS (1u << 7) /* keep the largest conflict-mark array L2-resident
                                              across batches: an L2 access-policy window
                                              (persisting set-aside sized from the device's L2)
                                              on the batch stream; result-identical            */
#define LTPG_FLAG_LOOPBACK_SHIFT 8         /* bits 8..11: logical partitions on one GPU   */
#define LTPG_FLAG_NO_SINGLE_LAUNCH (1u << 12) /* A/B: small single-partition OPS batches (<= 16384
                                              txns) normally run a2..a8 as ONE cooperative
                                              kernel with grid-wide barriers between the stages;
                                              this flag keeps them on the multi-kernel path     */

typedef struct {
  int device;                   /* CUDA device ordinal                                  */
  int rank, world;              /* partition of this process; world = 1: single GPU     */
  uint32_t max_txns;            /* per-batch capacity                                    */
  uint32_t max_ops;             /* OPS mode per-batch op capacity                         */
  uint32_t flags;               /* LTPG_FLAG_*                                           */
  uint32_t n_tables;            /* number of table ids used (<= 16)                      */
  uint32_t n_warehouses;        /* PROC mode: global TPC-C W (validation, routing; <= 1000) */
  uint64_t key_space;           /* OPS mode: keys [0, key_space) split into contiguous
                                   ranges over partitions (tables with owner_rule 2)      */
} ltpg_config;

/* Multi-GPU: world > 1 (<= 32) ranks each own a contiguous range of warehouses
 * (TPC-C, owner_rule 1) or of keys (OPS, owner_rule 2).  Global batches: every rank calls
 * ltpg_run_batch with the same global batch; each executes, marks and checks only the units it
 * owns, then the per-txn conflict bits are exchanged before write-back, so commit_bits / status
 * / abort_idx are identical on all ranks; result slots are filled by the owning rank and summed
 * over ranks.  The exchange runs over peer memory: each rank stores 4 bit planes per 32 txns
 * into every peer's exchange region over NVLink and raises a signal; the combine kernel waits
 * for all signals (no host round trip).  TPC-C can instead run SHARDED batches (ltpg_batch.grank,
 * see "Sharded batches"): each rank gets only the txns touching it, and only the bits of
 * cross-rank txns travel.  Bootstrap: every rank calls ltpg_peer_handle, the caller all-gathers
 * the handles (e.g. torch.distributed) and passes them, in rank order, to ltpg_connect_peers
 * before the first batch.  Every rank must run the same sequence of batches, and
 * ltpg_destroy_db only after every rank finished its last batch (a barrier): peers read
 * this rank's region during their batches.  A peer that never arrives fails the batch
 * after 20 s (LTPG_EINTERNAL).  LTPG_FLAG_LOOPBACK_SHIFT runs P logical partitions inside
 * one process on one GPU with the same ownership, combine and result-sum logic. */
#define LTPG_PEER_HANDLE_BYTES 128

typedef struct ltpg_db ltpg_db;  /* opaque, library-owned device state */

/* Create a database on config->device.  *out receives the handle. */
LTPG_API int ltpg_create_db(const ltpg_config* config, ltpg_db** out);

/* Peer-memory exchange bootstrap (world > 1).
 * ltpg_peer_handle writes this rank's LTPG_PEER_HANDLE_BYTES-byte handle (a CUDA IPC handle of
 * its exchange region plus the configuration it must match) to host memory `handle`.
 * ltpg_connect_peers takes all world handles back to back in rank order (host memory), checks
 * that every rank has the same max_txns / max_ops / flags (else EINVAL) and maps the peers'
 * regions.  Ranks on the same GPU are allowed (CUDA IPC within one device). */
LTPG_API int ltpg_peer_handle(ltpg_db* db, void* handle);
LTPG_API int ltpg_connect_peers(ltpg_db* db, const void* handles);

/* Table descriptor.  col_group[c] in [0, n_groups) or LTPG_STATIC; col_is_add[c]
 * marks a delayed-ADD column (its group may hold ADD columns only).  Tables with
 * static columns accept no DELETE; tables with n_groups == 0 accept no INSERT. */
typedef struct {
  uint32_t n_cols;              /* <= 16                                                 */
  const uint8_t* col_group;     /* host, n_cols                                          */
  const uint8_t* col_is_add;    /* host, n_cols                                          */
  uint32_t n_groups;            /* mutable column groups (conflict units per row), <= 15 */
  uint64_t capacity_rows;       /* rows incl. the append region                          */
  uint32_t has_pk;              /* 1: u64 primary key + hash index; 0: keyless (append)  */
  uint32_t owner_rule;          /* multi-GPU: 0 replicated, 1 TPC-C warehouse, 2 key range */
  uint32_t layout;              /* LTPG_LAYOUT_*: placement of the columns in HBM          */
} ltpg_table_desc;

/* Column placement (result-invisible).  ROWBLOCK: per row, the non-static
 * columns side by side and the static columns side by side (blocks of <= 8 words padded to
 * a power of two) -- for randomly accessed rows whose columns are used together.
 * COLUMNAR: one array per column -- for append-heavy tables written by consecutive lanes. */
enum { LTPG_LAYOUT_ROWBLOCK = 0, LTPG_LAYOUT_COLUMNAR = 1 };

/* Define table_id and load n_rows rows.  keys: host u64[n_rows] (NULL if keyless);
 * cols: host int64, column-major [n_cols][n_rows].  Duplicate keys -> EINVAL. */
LTPG_API int ltpg_load_table(ltpg_db* db, uint32_t table_id, const ltpg_table_desc* desc, uint64_t n_rows,
                    const uint64_t* keys, const int64_t* cols);

enum { LTPG_MODE_OPS = 0, LTPG_MODE_TPCC = 1 };

typedef struct {
  uint32_t n_txns;
  const uint64_t* tid;          /* [n_txns], strictly increasing (arrival order)  */
  uint32_t mode;                /* LTPG_MODE_OPS or LTPG_MODE_TPCC                       */
  uint32_t n_ops;               /* OPS: total ops                                         */
  const uint32_t* op_begin;     /* OPS: CSR [n_txns+1]                                    */
  const ltpg_op* ops;           /* OPS: [n_ops]                                           */
  const int64_t* op_arg;        /* OPS: [n_ops]                                           */
  const uint8_t* proc_type;     /* TPCC: [n_txns]                                         */
  const uint8_t* proc_params;   /* TPCC: [n_txns][128]                                    */
  int64_t batch_clock;          /* deterministic "now" for TPC-C dates                    */
  int inputs_on_device;         /* 1: the pointers above are device pointers             */
  void* stream;                 /* cudaStream_t to run on (NULL = legacy default)         */
  uint32_t flags;               /* LTPG_BATCH_*                                           */
  const uint32_t* proc_offsets; /* TPCC, optional [n_txns+1]: proc_params is PACKED -- txn r's
                                   block is bytes [off[r], off[r+1]) (<= 128, the used prefix
                                   of its 128-byte block; the rest reads as zero).  NULL: fixed
                                   128-byte blocks.  Cuts the host->device bytes ~2x.       */
  const uint32_t* grank;        /* TPCC, world > 1, optional [n_txns]: this is rank's SHARD of a
                                   global batch (see "Sharded batches" below): the global rank of
                                   each txn, strictly increasing, < n_global.  NULL: the batch is
                                   the global batch (every rank passes all of it).            */
  uint32_t n_global;            /* with grank: size of the global batch (<= max_txns)        */
} ltpg_batch;

/* Sharded batches (SURVEY §8(e) routing; world > 1, TPC-C): each rank receives only the txns
 * that touch its warehouses -- home warehouse, NewOrder supply warehouses, Payment customer
 * warehouse -- in global rank order, with their global ranks (ltpg_route_tpcc builds a rank's
 * shard from the global batch on the host).  The conflict TIDs are the global ranks, so every
 * unit's minimum marks are those of the whole batch.  Only the verdict bits of txns that touch
 * several ranks cross NVLink (one byte per txn and peer, stored into the peers' exchange regions),
 * plus the customer's (c_id, C_BALANCE) of a remote-customer Payment, returned to its home rank.
 * Outputs are per shard (index i = the shard's i-th txn): status / commit_bits / abort_idx for
 * every txn of the shard (identical on every rank that holds the txn); the result slots of a
 * txn are final on its home rank (the rank of its home warehouse). */

/* Inter-batch pipeline: with LTPG_BATCH_ASYNC, ltpg_run_batch enqueues the batch and
 * returns; host inputs are uploaded on an internal copy stream while the previous batch's
 * kernels run, and host outputs are downloaded on a second copy stream while the next batch's
 * kernels run.  At most three batches are in flight; ltpg_wait_batch(db, result) completes the
 * batch submitted with `result` and returns its status code.  Host buffers of an async batch
 * must stay valid (and unmodified) until then.  Batches still execute in submission order. */
#define LTPG_BATCH_ASYNC 1u
/* Compact TPC-C records (with proc_offsets; txn r's record is bytes [off[r], off[r+1])),
 * expanded to 128-byte blocks on the device -- ~1/2 the host->device bytes of used prefixes:
 * NewOrder   : u16 w | u8 d | u8 n_lines | u16 c | u8 rbk | u8 n_remote |
 *              n_lines x 22-bit line { i (bits 0-16) | qty-1 (bits 17-20) | remote (bit 21) },
 *              a little-endian bit stream (line l at bits 22 l .. 22 l + 21; ceil(22 n_lines / 8)
 *              bytes) | n_remote x u16 supply_w (of the remote lines, in line order; other
 *              lines are supplied by w)          = 8 + ceil(22 n_lines / 8) + 2 n_remote bytes
 * Payment    : bytes 0-11 of the block | u32 amount (0 <= amount < 2^32)  = 16 bytes
 * other types: the used prefix of the block (as without this flag).
 * A record whose length does not match its header is LTPG_EINVAL (nothing changed). */
#define LTPG_BATCH_COMPACT_PARAMS 2u
/* a9 on the device (TPC-C): the batch is the previous batch's conflict aborts -- kept on the
 * device with their original TIDs and parameter blocks, ascending ranks, never copied back to
 * the host -- followed by the n_txns txns given (host inputs, fixed or compact blocks, TIDs
 * larger than the carried ones).  The previous batch on this db must have completed (it is the
 * last one submitted; ltpg_wait_batch for an async one); ltpg_pending_aborts tells how many txns
 * it carries.  Outputs cover n_carried + n_txns txns (the carried ones first).  The previous
 * batch's device input and abort-list buffers (when they were the caller's) must stay valid until
 * this batch is submitted.  EINVAL: OPS mode, device inputs, a graph db, or no completed previous
 * batch, or n_carried + n_txns > max_txns. */
#define LTPG_BATCH_CARRY_ABORTS 4u
/* Consecutive TIDs (host inputs): `tid` points to ONE u64, the TID of the first given txn; the
 * i-th given txn has TID tid[0] + i (filled on the device, 8 bytes per txn less over PCIe).
 * With LTPG_BATCH_CARRY_ABORTS the carried txns keep their own TIDs (tid[0] must exceed them). */
#define LTPG_BATCH_TID_RANGE 8u

typedef struct {
  float ms_upload, ms_group, ms_exec, ms_detect, ms_exchange, ms_writeback, ms_download;
  uint32_t n_commit, n_conflict, n_user_abort;
  uint32_t n_kernels;           /* kernels this library launched for the batch */
  uint32_t popular_tables;      /* NEXT-3 (LTPG_FLAG_LARGE_BUCKETS): bit t = table t was popular in
                                   this batch (E = T/D > 1) and marked into large buckets */
} ltpg_stats;

typedef struct {
  uint32_t* commit_bits;        /* [ceil(n_txns/32)]: bit r%32 of word r/32 = committed   */
  uint8_t* status;              /* [n_txns]: LTPG_ST_*  (NULL with LTPG_RESULT_NO_STATUS) */
  uint32_t* abort_idx;          /* [n_txns] capacity: ranks of conflict aborts, ascending
                                   (NULL with LTPG_RESULT_NO_ABORT_LIST)                  */
  uint32_t* n_aborted;          /* [1]                                                    */
  int64_t* reads;               /* OPS: [n_ops]; TPCC: [4*n_txns]; NULL = not returned    */
  int outputs_on_device;        /* 1: the pointers above are device pointers             */
  ltpg_stats* stats;            /* optional host struct: per-stage device times           */
  uint32_t flags;               /* LTPG_RESULT_*                                          */
  uint64_t reads_cap;           /* capacity of `reads` in int64 slots (0: not checked); a
                                   batch that needs more (OPS: n_ops; TPCC: 4 x the txns it
                                   outputs, carried ones included) is LTPG_EINVAL before any
                                   state change                                           */
} ltpg_result;

/* Result options.  COMMITTED_READS (TPC-C): `reads` receives the 4 result slots of the COMMITTED
 * txns only, packed in rank order (the i-th committed txn -- the i-th set bit of commit_bits --
 * at reads[4i..4i+3]); a host `reads` buffer must be pinned and device-mapped (cudaHostAlloc;
 * the kernel writes it directly over PCIe, no copy of the other txns' slots), else EINVAL.
 * NO_STATUS / NO_ABORT_LIST: those outputs are not produced (their pointers may be NULL);
 * n_aborted and commit_bits always are.  Results of aborted txns are snapshot reads that are
 * recomputed when the txn is retried, so a closed loop needs only the committed ones. */
#define LTPG_RESULT_COMMITTED_READS 1u
#define LTPG_RESULT_NO_STATUS 2u
#define LTPG_RESULT_NO_ABORT_LIST 4u

/* Run one batch; synchronous on batch->stream (returns when results are in place)
 * unless batch->flags has LTPG_BATCH_ASYNC.
 * With LTPG_FLAG_GRAPH a single-process db (world == 1) runs a batch's device work (a2..a8:
 * every kernel, memset and intra-batch stream fork/join) as one CUDA graph: the first batch of
 * a shape is captured and instantiated (slow: ~0.1-2 ms of host time), later batches of the same
 * shape (n_txns, n_ops, input/output pointers when on the device, flags) replay it; epoch and
 * clock reach the kernels through device memory.  Up to four shapes are kept per pipeline
 * slot.  Results are identical either way. */
LTPG_API int ltpg_run_batch(ltpg_db* db, const ltpg_batch* batch, ltpg_result* result);

/* Complete an asynchronously submitted batch (see LTPG_BATCH_ASYNC). */
LTPG_API int ltpg_wait_batch(ltpg_db* db, ltpg_result* result);

/* Number of conflict aborts an LTPG_BATCH_CARRY_ABORTS batch submitted now would carry (those of
 * the last batch, once it completed; 0 if there is none or it is still in flight). */
LTPG_API int ltpg_pending_aborts(ltpg_db* db, uint32_t* n_aborted);

/* NEXT-3 / Table VIII: bytes of table t's conflict marks -- standard-sized (one word per
 * unit and kind) and large-sized buckets (LTPG_FLAG_LARGE_BUCKETS), as allocated -- and the bucket
 * size s_u allocated (1: none).  Host outputs; EINVAL for a bad table id. */
LTPG_API int ltpg_mark_memory(ltpg_db* db, uint32_t table_id, uint64_t* standard_bytes, uint64_t* large_bytes,
                              uint32_t* su);

/* Canonical dump (valid rows only): keyed tables sorted by key, keyless tables by
 * the full column tuple.  Call with keys == cols == NULL to get *n_rows only.
 * keys: host u64[n_rows]; cols: host int64 [n_cols][n_rows]. */
LTPG_API int ltpg_dump_table(ltpg_db* db, uint32_t table_id, uint64_t* n_rows, uint64_t* keys, int64_t* cols);

/* ---- a9: the host retry loop ("aborted transactions ... are re-executed in the next
 * batch", P:120 TID order) ------------------------------------------------------------------
 * The next batch = the conflict aborts of `prev` (abort_idx as returned by ltpg_run_batch:
 * ascending ranks), with their original TIDs and inputs, followed by a prefix of `fresh`, as
 * many fresh txns as fit in out->cap_txns (and, OPS, out->cap_ops).  Because every aborted TID is
 * smaller than every fresh one, the retried txns take the smallest ranks: the batch's smallest
 * rank commits unless it user-aborts, so no txn is retried forever.
 * Host memory only (prev/fresh with inputs_on_device == 0 and fixed 128-byte TPC-C blocks; the
 * caller owns every buffer).  Needs no db and no GPU.  Errors (EINVAL, nothing written
 * past the buffers): mode mismatch, device or packed inputs, an abort index out of range or
 * not ascending, the aborts alone exceeding the capacity, or a fresh TID not larger than the
 * last retried one. */
typedef struct {
  uint32_t cap_txns, cap_ops;   /* in: capacity of the buffers below (txns / OPS ops)       */
  uint64_t* tid;                /* [cap_txns]                                               */
  uint32_t* op_begin;           /* OPS: [cap_txns+1]                                        */
  ltpg_op* ops;                 /* OPS: [cap_ops]                                           */
  int64_t* op_arg;              /* OPS: [cap_ops]                                           */
  uint8_t* proc_type;           /* TPCC: [cap_txns]                                         */
  uint8_t* proc_params;         /* TPCC: [cap_txns][128]                                    */
  uint32_t n_txns, n_ops;       /* out: the composed batch                                  */
  uint32_t n_retried, n_fresh;  /* out: aborts carried over, fresh txns taken (a prefix)    */
} ltpg_batch_buf;
LTPG_API int ltpg_compose_retry(const ltpg_batch* prev, const uint32_t* abort_idx, uint32_t n_aborted,
                                const ltpg_batch* fresh, ltpg_batch_buf* out);

/* Routing (host, no db or GPU needed): the shard of `rank` out of the global TPC-C batch
 * `global` (host memory, fixed 128-byte blocks) for `world` ranks owning contiguous ranges of
 * n_warehouses warehouses: the txns whose home / supply / customer warehouse the rank owns, in
 * order, copied into out (tid, proc_type, proc_params) with their global ranks in grank[cap_txns];
 * out->n_txns receives the shard size.  EINVAL: bad arguments or capacity too small. */
LTPG_API int ltpg_route_tpcc(const ltpg_batch* global, uint32_t n_warehouses, uint32_t world, uint32_t rank,
                             ltpg_batch_buf* out, uint32_t* grank);


LTPG_API void ltpg_destroy_db(ltpg_db* db);
LTPG_API const char* ltpg_last_error(const ltpg_db* db);
/* Library version string, e.g. "ltpg-b200 0.1 sm_100a". */
LTPG_API const char* ltpg_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LTPG_H */
