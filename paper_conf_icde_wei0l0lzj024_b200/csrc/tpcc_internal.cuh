// TPC-C PROC-mode scratch and launchers (pre-compiled stored procedures).
#pragma once
#include "ltpg_internal.cuh"
#include "small.cuh"

namespace ltpg {

constexpr int NTYPES = 5;
constexpr int TLOG = 20;         // u32 row slots logged per txn by execute (NewOrder 16, Payment 4,
                                 // OrderStatus 17), padded to 80 B so every txn's log is 16-B aligned
constexpr int NO_CHUNK = 1024;   // ranks per chunk of the o_id prefix computation
constexpr int SMALL_CHUNK = 32;  // the same on the single-launch path (k_tpcc_small)

// TPC-C schema (include/ltpg.h): table ids and column indices
enum { TW = 0, TD = 1, TC = 2, TH = 3, TNO = 4, TO = 5, TOL = 6, TI = 7, TS = 8 };
enum { W_TAX = 0, W_YTD = 1 };
enum { D_TAX = 0, D_YTD = 1, D_NEXT_O_ID = 2, D_NEXT_DELIV_O_ID = 3 };
enum { C_DISCOUNT = 0, C_CREDIT = 1, C_LAST = 2, C_FIRST = 3, C_INIT_O_ID = 4, C_BALANCE = 5,
       C_YTD_PAYMENT = 6, C_PAYMENT_CNT = 7, C_DELIVERY_CNT = 8 };
enum { H_C_ID = 0, H_C_D_ID, H_C_W_ID, H_D_ID, H_W_ID, H_DATE, H_AMOUNT, H_TID, H_SEQ };
enum { NO_O_ID = 0 };
enum { O_C_ID = 0, O_ENTRY_D = 1, O_OL_CNT = 2, O_ALL_LOCAL = 3, O_CARRIER_ID = 4 };
enum { OL_I_ID = 0, OL_SUPPLY_W_ID = 1, OL_QUANTITY = 2, OL_AMOUNT = 3, OL_DELIVERY_D = 4 };
enum { I_PRICE = 0, I_IM_ID = 1 };
enum { S_QUANTITY = 0, S_YTD = 1, S_ORDER_CNT = 2, S_REMOTE_CNT = 3 };

// counters in TpccDev::misc (M_NO / M_NO_LINES / M_PAY: inserts this partition may append)
// M_DONE_G / M_DONE_WB: blocks of k_tpcc_group / the write-back phase that finished (the last
// one runs the capacity check / the row-counter advance)
enum { M_HIST = 0, M_NO_LINES = 1, M_PAY = 2, M_NO = 3, M_DONE_G = 4, M_DONE_WB = 5, M_CCOUNT = 8 };

// StockLevel shared per district (k_sl_*): per-batch scratch indexed by district key (dk) or by
// the compact index of a district with StockLevels in the batch (idx)
struct SlScratch {
  uint32_t* minr = nullptr;     // [dsz] by dk: smallest StockLevel rank (0xFFFFFFFF: none)
  uint32_t* slot = nullptr;     // [dsz] by dk: idx
  uint32_t* dk = nullptr;       // [dsz] by idx
  uint32_t* cnt = nullptr;      // [1] listed districts
  uint32_t* low = nullptr;      // [dsz][257] by idx: #distinct items with S_QUANTITY < t
  long long* nx = nullptr;      // [dsz] by idx: D_NEXT_O_ID
  uint32_t* rows = nullptr;     // [dsz][300] by idx: stock rows of the distinct items
  uint32_t* nd = nullptr;       // [dsz] by idx: distinct items
  uint32_t* rowd = nullptr;     // [dsz] by idx: district row
  uint32_t* m = nullptr;        // [dsz] by idx: smallest write/add mark rank over the unit set
};

struct TpccDev {
  uint32_t max_txns = 0;
  uint32_t nw = 0;              // n_warehouses (global)
  uint32_t dsz = 0;             // district-key array size = nw*10 + 11
  int* by_name = nullptr;       // dense secondary index [(w*10+d)*1000 + c_last] -> c_id (0: none)
  bool owns_by_name = false;    // loopback partitions share partition 0's index
  uint32_t* list = nullptr;     // [NTYPES][max_txns] ranks, grouped by procedure type
  uint32_t* clist = nullptr;    // [NTYPES][max_txns] committed ranks (write-back only)
  uint32_t* log = nullptr;      // [max_txns][TLOG] rows found by execute
  unsigned long long* no_pref = nullptr;  // [max_txns+1] committed NewOrder (lines << 32 | 1) -> exclusive scan
  uint32_t* dk_of = nullptr;    // [max_txns] district key of a committed NewOrder, else ~0
  uint32_t* chunk_cnt = nullptr;// [chunks][dsz]
  long long* dist_base = nullptr; // [dsz] snapshot D_NEXT_O_ID
  unsigned long long* chunk_tot = nullptr;  // [chunks+1] committed NewOrder (lines << 32 | 1) per chunk -> bases
  uint32_t* dl_min = nullptr;   // [nw+1] smallest Delivery rank per warehouse this batch (~0: none)
  uint32_t* misc = nullptr;     // counters (M_*)
  SlScratch sl;
  cudaStream_t side = nullptr;  // StockLevel phases run here, concurrently with the others
  cudaEvent_t fork[2]{}, join[2]{};
  const DevTable* h_tab = nullptr; // host table copies (NEXT-3 bucket reduce between exec and detect)
  uint32_t n_tab = 0;
  uint16_t* d_su = nullptr;        // NEXT-3: this batch's bucket size per table (capi.cu)
  uint32_t* popular = nullptr;     // NEXT-3: bitmask of this batch's popular tables (set per batch)
};

struct TpccParams {
  uint32_t* clist;              // committed re-list target (k_tpcc_relist)
  uint32_t* list;
  const uint32_t* counts;       // per-type list lengths of `list` (kcount, or misc + M_CCOUNT)
  uint32_t* log;
  unsigned long long* no_pref;  // exclusive prefix: low 32 = committed NewOrders, high 32 = their lines
  uint32_t* dk_of;
  uint32_t* chunk_cnt;
  long long* dist_base;
  uint32_t* misc;
  const int* by_name;
  uint32_t nw, dsz, max_txns, n_chunks;
  unsigned long long* chunk_tot;
  uint32_t* dl_min;
  uint32_t agg_dsz;             // write-back: DISTRICT D_YTD deltas aggregated per block (0: not)
  uint32_t hot_words;           // execute: shared-memory marks of the W / D units (nw + 30 nw; 0: off)
  uint32_t chunk_shift;         // log2 ranks per o_id chunk (NO_CHUNK; SMALL_CHUNK on the single-launch path)
  bool oid_inline;              // write-back computes the o_id (single-launch path, no k_no_assign)
  bool cc_dm;                   // chunk_cnt district-major (dsz <= COLSCAN_TILED_DSZ, single-launch path)
};
constexpr uint32_t COLSCAN_TILED_DSZ = 2048;  // above: chunk-major chunk counts, k_no_colscan_tiled

int tpcc_alloc(TpccDev& t, uint32_t max_txns, uint32_t n_warehouses, int* shared_by_name);
void tpcc_free(TpccDev& t);
int tpcc_build_secondary(TpccDev& t, const uint64_t* keys, const int64_t* cols, uint64_t n_rows,
                         uint32_t n_warehouses);
// front: validate + lists, capacity, execute, detect;  back: o_id prefix, write-back, cursors
int tpcc_front(TpccDev& t, BatchDev& b, cudaStream_t s, cudaEvent_t* ev, bool cleared);
int tpcc_back(TpccDev& t, BatchDev& b, uint32_t* scan_scratch, cudaStream_t s);
// single-launch path for small single-partition batches (k_tpcc_small): n_txns <= max_txns()
// and n_warehouses <= TPCC_SMALL_MAX_W (the per-warp o_id counters live in shared memory);
// tpcc_small_clear puts the batch scratch into the rest state the kernel expects (after a
// multi-kernel batch, which leaves it dirty)
constexpr uint32_t TPCC_SMALL_MAX_W = 64;
uint32_t tpcc_small_max_txns();
bool tpcc_small_fits(const TpccDev& t);
void tpcc_small_clear(TpccDev& t, cudaStream_t s);
int launch_tpcc_small(TpccDev& t, const BatchDev& b, const SmallOut& o, cudaStream_t s);
// ORDER.aux[row] = first row of the order's ORDER_LINE rows when they are contiguous
void tpcc_build_olrow(cudaStream_t s);

}  // namespace ltpg
