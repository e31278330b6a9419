// LTPG CPU ORACLE -- TEST INFRASTRUCTURE ONLY.
//
// A plain, slow implementation of one LTPG batch under
// deterministic optimistic concurrency control (§IV, Alg. 1
// P:128-157), written from the paper and the readings in DESIGN.md.  Only
// tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
// reference legs may load this library.  It shares no code, header, constant
// or helper with the CUDA path (paper_conf_icde_wei0l0lzj024_b200/csrc).
//
// What it computes, in the paper's order:
//   O1 execute   (P:104, P:106, P:122, P:146 readMem/recordLS): every txn runs
//                against the pre-batch snapshot S; writes are buffered locally.
//   O2 marks     ("each transaction must register its TIDs", P:203,
//                P:225 atomicMin => per-unit minimum): minR/minW/minA over ALL
//                txns of the batch, including ones that will abort (R2).
//   O3 commit    (P:108, P:147-151 rcheck/wcheck, P:80 Aria rule; R1):
//                abort iff RAW or WAW against a smaller TID:
//                  exists u in RS u WS : min(minW[u], minA[u]) < r
//                  exists u in AS      : minW[u] < r           (R7: ADD-ADD commute)
//   O4 apply     (P:152-157 writeMem): committed write sets in TID order;
//                delayed adds accumulate, fetch pre-images in TID order.
//   O5 output    status / reads / canonical table dump.
// Conflict unit = (table, key, column group) (R4, P:239 row-level splitting).
//
// Single-threaded by default.  orc_set_threads(h, T > 1) is the SURVEY §8(d) secondary CPU
// baseline: O1 runs over txns on T std::threads (every txn reads only the snapshot), O2 / O3
// shard the conflict units over the threads by hash (each thread builds the min marks of its
// own units, then tests the txns of a contiguous rank range against them); O4 stays serial.
// tests/test_oracle_threads.py checks that it equals the single-threaded run.
//
// Parity: pinned by tests/test_oracle_*.py (Example 2/3 of the paper, brute
// force of the pairwise definition, serial replay, TPC-C consistency
// conditions, Table VI "no" rows, closed forms).
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <map>
#include <thread>
#include <unordered_map>
#include <unordered_set>
#include <vector>

namespace {

constexpr int64_t NOT_FOUND = INT64_MIN;
constexpr uint8_t STATIC_GROUP = 0xFF;
constexpr uint16_t COL_COUNT = 0xFFFF;
constexpr uint64_t KEY_RESERVED = ~0ull;
enum : uint8_t { K_SELECT = 0, K_UPDATE = 1, K_ADD = 2, K_INSERT = 3, K_DELETE = 4, K_SCAN = 5 };
enum : uint8_t { ACC_R = 0, ACC_W = 1, ACC_A = 2 };
enum : uint8_t { ST_CONFLICT = 0, ST_COMMIT = 1, ST_USER_ABORT = 2 };
enum { ORC_OK = 0, ORC_EINVAL = -1, ORC_EINTERNAL = -7 };

struct Table {
  bool defined = false;
  uint32_t n_cols = 0, n_groups = 0;
  bool has_pk = false;
  std::vector<uint8_t> group, is_add;
  std::vector<std::vector<int64_t>> col;  // col[c][row]
  std::vector<uint64_t> key;              // key[row]
  std::vector<uint8_t> valid;             // hidden existence column
  std::unordered_map<uint64_t, uint64_t> pk;  // key -> row, valid rows only
  uint64_t rows() const { return valid.size(); }
  bool find(uint64_t k, uint64_t* row) const {
    auto it = pk.find(k);
    if (it == pk.end()) return false;
    *row = it->second;
    return true;
  }
  uint64_t append(uint64_t k, const std::vector<int64_t>& vals) {
    uint64_t r = valid.size();
    for (uint32_t c = 0; c < n_cols; ++c) col[c].push_back(vals[c]);
    key.push_back(k);
    valid.push_back(1);
    if (has_pk) pk[k] = r;
    return r;
  }
};

struct Unit {
  uint32_t t;
  uint32_t g;
  uint64_t key;
  bool operator==(const Unit& o) const { return t == o.t && g == o.g && key == o.key; }
};
struct UnitHash {
  size_t operator()(const Unit& u) const {
    uint64_t h = u.key * 0x9E3779B97F4A7C15ull ^ (uint64_t(u.t) << 40) ^ (uint64_t(u.g) << 56);
    return size_t(h ^ (h >> 29));
  }
};
struct Access {
  Unit u;
  uint8_t acc;
};

// Buffered write set entry (recordLS), applied at write-back (writeMem).
enum : uint8_t { E_SET = 0, E_ADD = 1, E_INSERT = 2, E_DELETE = 3, E_APPEND = 4 };
struct Effect {
  uint8_t kind;
  uint32_t t;
  uint64_t key;
  uint32_t c;
  int64_t v;
  std::vector<int64_t> vals;  // INSERT / APPEND
};

struct TxnExec {
  std::vector<Access> acc;
  std::vector<Effect> eff;
  bool user_abort = false;
  // TPC-C NewOrder deferred part (fetch-ADD of D_NEXT_O_ID, P:241 / R12)
  bool is_neworder = false;
  uint64_t no_dkey = 0;
  std::vector<std::vector<int64_t>> ol_vals;  // per line: OL_* columns
  std::vector<int64_t> o_vals;                // ORDER columns
};

struct Db {
  std::vector<Table> tables;
  uint32_t n_warehouses = 0;
  // TPC-C static secondary index (w,d,last) -> c_id ("secondary hash tables")
  std::unordered_map<uint64_t, int64_t> by_name;
  bool by_name_built = false;
  std::vector<double> stage_ns;
  bool reorder = false;  // NEXT-1 logical reordering
  unsigned threads = 1;  // SURVEY §8(d) secondary baseline (orc_set_threads)
};

// Run f(lo, hi) over [0, n) split into T contiguous ranges on T threads.
template <class F>
void parallel_ranges(uint32_t n, unsigned T, F f) {
  if (T <= 1 || n < 2 * T) {
    f(0u, n);
    return;
  }
  std::vector<std::thread> th;
  for (unsigned k = 0; k < T; ++k)
    th.emplace_back([&, k] { f(uint32_t(uint64_t(n) * k / T), uint32_t(uint64_t(n) * (k + 1) / T)); });
  for (auto& t : th) t.join();
}

// ---------------------------------------------------------------------------
// O2 + O3: marks and the commit rule.
// ---------------------------------------------------------------------------
//   reorder = false (hot path, R1):  abort iff WAW or RAW
//   reorder = true  (NEXT-1, logical reordering P:237 / Aria P:80):  abort iff WAW or (RAW and WAR)
// with, for txn r:
//   WAW: a unit r writes was written or added to by a smaller rank, or a unit r adds to was
//        plainly written by a smaller rank (ADD-ADD commute, R7)
//   RAW: a unit r reads was written or added to by a smaller rank
//   WAR: a unit r writes or adds to was read by a smaller rank
void decide(const std::vector<TxnExec>& ex, std::vector<uint8_t>& status, bool reorder) {
  const uint32_t n = ex.size();
  std::unordered_map<Unit, uint32_t, UnitHash> minR, minW, minA;  // P:219 "two kinds of TIDs"
  auto mark = [](std::unordered_map<Unit, uint32_t, UnitHash>& m, const Unit& u, uint32_t r) {
    auto it = m.find(u);
    if (it == m.end()) m.emplace(u, r);
    else if (r < it->second) it->second = r;  // atomicMin
  };
  for (uint32_t r = 0; r < n; ++r)
    for (const Access& a : ex[r].acc) {
      if (a.acc == ACC_R) mark(minR, a.u, r);
      else if (a.acc == ACC_W) mark(minW, a.u, r);
      else mark(minA, a.u, r);
    }
  auto get = [](const std::unordered_map<Unit, uint32_t, UnitHash>& m, const Unit& u) -> uint32_t {
    auto it = m.find(u);
    return it == m.end() ? UINT32_MAX : it->second;
  };
  status.assign(n, ST_COMMIT);
  for (uint32_t r = 0; r < n; ++r) {
    bool waw = false, raw = false, war = false;
    for (const Access& a : ex[r].acc) {
      const uint32_t w = get(minW, a.u), ad = get(minA, a.u), rd = get(minR, a.u);
      if (a.acc == ACC_R) {
        if (std::min(w, ad) < r) raw = true;
      } else if (a.acc == ACC_W) {
        if (std::min(w, ad) < r) waw = true;
        if (rd < r) war = true;
      } else {
        if (w < r) waw = true;
        if (rd < r) war = true;
      }
    }
    const bool abort = reorder ? (waw || (raw && war)) : (waw || raw);
    status[r] = abort ? ST_CONFLICT : (ex[r].user_abort ? ST_USER_ABORT : ST_COMMIT);
  }
}

// The same O2 + O3 with T threads: thread k builds the min marks of the units u with
// hash(u) % T == k (over all txns, in any order: min is order-free), then every thread tests
// the txns of its rank range against the shard maps (read-only).  Identical to decide().
void decide_threads(const std::vector<TxnExec>& ex, std::vector<uint8_t>& status, bool reorder, unsigned T) {
  const uint32_t n = ex.size();
  using Map = std::unordered_map<Unit, uint32_t, UnitHash>;
  std::vector<Map> minR(T), minW(T), minA(T);
  UnitHash H;
  std::vector<std::thread> th;
  for (unsigned k = 0; k < T; ++k)
    th.emplace_back([&, k] {
      for (uint32_t r = 0; r < n; ++r)
        for (const Access& a : ex[r].acc) {
          if (H(a.u) % T != k) continue;
          Map& m = a.acc == ACC_R ? minR[k] : (a.acc == ACC_W ? minW[k] : minA[k]);
          auto it = m.find(a.u);
          if (it == m.end()) m.emplace(a.u, r);
          else if (r < it->second) it->second = r;
        }
    });
  for (auto& t : th) t.join();
  auto get = [&](const std::vector<Map>& ms, const Unit& u) -> uint32_t {
    const Map& m = ms[H(u) % T];
    auto it = m.find(u);
    return it == m.end() ? UINT32_MAX : it->second;
  };
  status.assign(n, ST_COMMIT);
  parallel_ranges(n, T, [&](uint32_t lo, uint32_t hi) {
    for (uint32_t r = lo; r < hi; ++r) {
      bool waw = false, raw = false, war = false;
      for (const Access& a : ex[r].acc) {
        const uint32_t w = get(minW, a.u), ad = get(minA, a.u), rd = get(minR, a.u);
        if (a.acc == ACC_R) {
          if (std::min(w, ad) < r) raw = true;
        } else if (a.acc == ACC_W) {
          if (std::min(w, ad) < r) waw = true;
          if (rd < r) war = true;
        } else {
          if (w < r) waw = true;
          if (rd < r) war = true;
        }
      }
      const bool abort = reorder ? (waw || (raw && war)) : (waw || raw);
      status[r] = abort ? ST_CONFLICT : (ex[r].user_abort ? ST_USER_ABORT : ST_COMMIT);
    }
  });
}

// O4: apply one buffered effect (writeMem).
int apply_effect(Db& db, const Effect& e) {
  Table& T = db.tables[e.t];
  uint64_t row;
  switch (e.kind) {
    case E_SET:
      if (!T.find(e.key, &row)) return ORC_EINTERNAL;
      T.col[e.c][row] = e.v;
      return ORC_OK;
    case E_ADD:
      if (!T.find(e.key, &row)) return ORC_EINTERNAL;
      T.col[e.c][row] = int64_t(uint64_t(T.col[e.c][row]) + uint64_t(e.v));  // wrap-around (R9)
      return ORC_OK;
    case E_INSERT:
      if (T.pk.count(e.key)) return ORC_EINTERNAL;
      T.append(e.key, e.vals);
      return ORC_OK;
    case E_APPEND:
      T.append(0, e.vals);
      return ORC_OK;
    case E_DELETE:
      if (!T.find(e.key, &row)) return ORC_EINTERNAL;
      T.valid[row] = 0;
      T.pk.erase(e.key);
      return ORC_OK;
  }
  return ORC_EINTERNAL;
}

// ---------------------------------------------------------------------------
// OPS mode (YCSB and hand-written micro-cases).  Op record: 16 bytes
//   u64 key | u8 kind | u8 table | u16 col | u32 aux      (include/ltpg.h)
// ---------------------------------------------------------------------------
struct Op {
  uint64_t key;
  uint8_t kind, table;
  uint16_t col;
  uint32_t aux;
};
Op read_op(const uint8_t* p) {
  Op o;
  std::memcpy(&o.key, p, 8);
  o.kind = p[8];
  o.table = p[9];
  std::memcpy(&o.col, p + 10, 2);
  std::memcpy(&o.aux, p + 12, 4);
  return o;
}
bool is_write_kind(uint8_t k) { return k == K_UPDATE || k == K_ADD || k == K_INSERT || k == K_DELETE; }

int validate_ops(const Db& db, uint32_t n, const uint64_t* tid, const uint32_t* ob, const uint8_t* ops) {
  for (uint32_t r = 1; r < n; ++r)
    if (tid[r] <= tid[r - 1]) return ORC_EINVAL;  // TIDs by arrival, unique
  if (n && ob[0] != 0) return ORC_EINVAL;
  for (uint32_t r = 0; r < n; ++r) {
    if (ob[r + 1] < ob[r]) return ORC_EINVAL;
    for (uint32_t i = ob[r]; i < ob[r + 1]; ++i) {
      Op o = read_op(ops + 16ull * i);
      if (o.table >= db.tables.size() || !db.tables[o.table].defined) return ORC_EINVAL;
      const Table& T = db.tables[o.table];
      if (!T.has_pk || o.kind > K_SCAN || o.key == KEY_RESERVED) return ORC_EINVAL;
      switch (o.kind) {
        case K_SELECT:
          if (o.col >= T.n_cols) return ORC_EINVAL;
          break;
        case K_UPDATE:
          if (o.col >= T.n_cols || T.group[o.col] == STATIC_GROUP || T.is_add[o.col]) return ORC_EINVAL;
          break;
        case K_ADD:
          if (o.col >= T.n_cols || !T.is_add[o.col]) return ORC_EINVAL;
          break;
        case K_INSERT:
          if (T.n_groups == 0) return ORC_EINVAL;
          break;
        case K_DELETE: {
          if (T.n_groups == 0) return ORC_EINVAL;
          for (uint32_t c = 0; c < T.n_cols; ++c)
            if (T.group[c] == STATIC_GROUP) return ORC_EINVAL;
          break;
        }
        case K_SCAN:
          if (o.col != COL_COUNT && o.col >= T.n_cols) return ORC_EINVAL;
          if (o.aux > 0 && o.key > KEY_RESERVED - o.aux) return ORC_EINVAL;
          break;
      }
    }
    // R10: a key written by a txn is touched by no other op of that txn
    for (uint32_t i = ob[r]; i < ob[r + 1]; ++i)
      for (uint32_t j = ob[r]; j < i; ++j) {
        Op a = read_op(ops + 16ull * i), b = read_op(ops + 16ull * j);
        if (a.table != b.table) continue;
        uint64_t alo = a.key, ahi = a.kind == K_SCAN ? a.key + a.aux : a.key + 1;
        uint64_t blo = b.key, bhi = b.kind == K_SCAN ? b.key + b.aux : b.key + 1;
        bool overlap = alo < bhi && blo < ahi;
        if (!overlap) continue;
        if (is_write_kind(a.kind) || is_write_kind(b.kind)) return ORC_EINVAL;
        if (a.kind != K_SCAN && b.kind != K_SCAN) return ORC_EINVAL;  // duplicate point key
      }
  }
  return ORC_OK;
}

// O1 for one op: snapshot read (readMem), local write buffering (recordLS),
// access registration for the marks (recordTID).
void exec_op(const Db& db, const Op& o, int64_t arg, TxnExec& tx, int64_t* res) {
  const Table& T = db.tables[o.table];
  uint64_t row;
  bool present = T.find(o.key, &row);
  auto unit = [&](uint64_t k, uint32_t g) { return Unit{o.table, g, k}; };
  auto exist_read = [&](uint64_t k) {  // absent key: READ of the key's (existence) unit
    if (T.n_groups) tx.acc.push_back({unit(k, 0), ACC_R});
  };
  switch (o.kind) {
    case K_SELECT:
      if (!present) { *res = NOT_FOUND; exist_read(o.key); return; }
      *res = T.col[o.col][row];
      if (T.group[o.col] != STATIC_GROUP) tx.acc.push_back({unit(o.key, T.group[o.col]), ACC_R});
      return;
    case K_UPDATE:  // read-modify-write v <- v + arg (SURVEY §8(c) YCSB)
      if (!present) { *res = NOT_FOUND; exist_read(o.key); return; }
      *res = T.col[o.col][row];
      tx.acc.push_back({unit(o.key, T.group[o.col]), ACC_W});
      tx.eff.push_back({E_SET, o.table, o.key, o.col, int64_t(uint64_t(*res) + uint64_t(arg)), {}});
      return;
    case K_ADD:  // delayed blind add
      if (!present) { *res = NOT_FOUND; exist_read(o.key); return; }
      *res = 0;
      tx.acc.push_back({unit(o.key, T.group[o.col]), ACC_A});
      tx.eff.push_back({E_ADD, o.table, o.key, o.col, arg, {}});
      return;
    case K_INSERT:
      if (present) {  // duplicate key: user abort, counts as a READ
        *res = 0;
        tx.user_abort = true;
        tx.acc.push_back({unit(o.key, 0), ACC_R});
        return;
      }
      *res = 1;
      for (uint32_t g = 0; g < T.n_groups; ++g) tx.acc.push_back({unit(o.key, g), ACC_W});
      {
        Effect e{E_INSERT, o.table, o.key, 0, 0, {}};
        for (uint32_t c = 0; c < T.n_cols; ++c) e.vals.push_back(int64_t(uint64_t(arg) + c));
        tx.eff.push_back(e);
      }
      return;
    case K_DELETE:
      if (!present) { *res = NOT_FOUND; exist_read(o.key); return; }
      *res = 1;
      for (uint32_t g = 0; g < T.n_groups; ++g) tx.acc.push_back({unit(o.key, g), ACC_W});
      tx.eff.push_back({E_DELETE, o.table, o.key, 0, 0, {}});
      return;
    case K_SCAN: {  // contiguous key range [key, key+len) (R8); phantom-safe
      int64_t cnt = 0;
      uint64_t sum = 0;
      for (uint64_t k = o.key; k < o.key + o.aux; ++k) {
        uint64_t rr;
        if (T.find(k, &rr)) {
          ++cnt;
          if (o.col != COL_COUNT) sum += uint64_t(T.col[o.col][rr]);
          uint32_t g = (o.col != COL_COUNT && T.group[o.col] != STATIC_GROUP) ? T.group[o.col] : 0;
          if (T.n_groups) tx.acc.push_back({unit(k, g), ACC_R});
        } else {
          exist_read(k);
        }
      }
      *res = o.col == COL_COUNT ? cnt : int64_t(sum);
      return;
    }
  }
}

// ---------------------------------------------------------------------------
// PROC mode: TPC-C stored procedures, integer-only.
// Table ids / column order: include/ltpg.h "TPC-C schema" (restated here).
// ---------------------------------------------------------------------------
enum { TW = 0, TD = 1, TC = 2, TH = 3, TNO = 4, TO = 5, TOL = 6, TI = 7, TS = 8 };
enum { W_TAX = 0, W_YTD = 1 };
enum { D_TAX = 0, D_YTD = 1, D_NEXT_O_ID = 2, D_NEXT_DELIV_O_ID = 3 };
enum { C_DISCOUNT = 0, C_CREDIT = 1, C_LAST = 2, C_FIRST = 3, C_INIT_O_ID = 4, C_BALANCE = 5,
       C_YTD_PAYMENT = 6, C_PAYMENT_CNT = 7, C_DELIVERY_CNT = 8 };
enum { O_C_ID = 0, O_ENTRY_D = 1, O_OL_CNT = 2, O_ALL_LOCAL = 3, O_CARRIER_ID = 4 };
enum { OL_I_ID = 0, OL_SUPPLY_W_ID = 1, OL_QUANTITY = 2, OL_AMOUNT = 3, OL_DELIVERY_D = 4 };
enum { I_PRICE = 0 };
enum { S_QUANTITY = 0, S_YTD = 1, S_ORDER_CNT = 2, S_REMOTE_CNT = 3 };
enum { P_NEWORDER = 0, P_PAYMENT = 1, P_ORDERSTATUS = 2, P_DELIVERY = 3, P_STOCKLEVEL = 4 };

uint64_t key_d(uint64_t w, uint64_t d) { return w * 10 + d; }
uint64_t key_c(uint64_t w, uint64_t d, uint64_t c) { return key_d(w, d) * 3000 + c; }
uint64_t key_s(uint64_t w, uint64_t i) { return w * 100000 + i; }
uint64_t key_o(uint64_t w, uint64_t d, uint64_t o) { return (key_d(w, d) << 32) | o; }
uint64_t key_ol(uint64_t w, uint64_t d, uint64_t o, uint64_t ol) { return key_o(w, d, o) * 16 + ol; }

template <class T> T rd(const uint8_t* p, int off) { T v; std::memcpy(&v, p + off, sizeof(T)); return v; }

struct ProcCtx {
  const Db& db;
  TxnExec& tx;
  int64_t clock;
  uint64_t tid;
  bool ok = true;
  int64_t get(uint32_t t, uint64_t k, uint32_t c) {
    uint64_t row;
    if (!db.tables[t].find(k, &row)) { ok = false; return 0; }
    return db.tables[t].col[c][row];
  }
  bool exists(uint32_t t, uint64_t k) { uint64_t row; return db.tables[t].find(k, &row); }
  uint8_t grp(uint32_t t, uint32_t c) const { return db.tables[t].group[c]; }
  bool add_col(uint32_t t, uint32_t c) const { return db.tables[t].is_add[c]; }
  // mark a read of column c (static columns are never written: unmarked, R4)
  void rd_mark(uint32_t t, uint64_t k, uint32_t c) {
    if (grp(t, c) != STATIC_GROUP) tx.acc.push_back({Unit{t, grp(t, c), k}, ACC_R});
  }
  void acc(uint32_t t, uint64_t k, uint32_t g, uint8_t a) { tx.acc.push_back({Unit{t, g, k}, a}); }
  void set(uint32_t t, uint64_t k, uint32_t c, int64_t v) { tx.eff.push_back({E_SET, t, k, c, v, {}}); }
  void add(uint32_t t, uint64_t k, uint32_t c, int64_t v) { tx.eff.push_back({E_ADD, t, k, c, v, {}}); }
  // Update column group of (t,k): strict -> WRITE unit with buffered new values;
  // delayed (ADD columns) -> ADD unit with deltas.
  void upd_add(uint32_t t, uint64_t k, uint32_t c, int64_t delta) {
    if (add_col(t, c)) {
      acc(t, k, grp(t, c), ACC_A);
      add(t, k, c, delta);
    } else {
      acc(t, k, grp(t, c), ACC_W);
      set(t, k, c, int64_t(uint64_t(get(t, k, c)) + uint64_t(delta)));
    }
  }
};

int64_t lookup_by_name(const Db& db, uint64_t w, uint64_t d, uint64_t last) {
  auto it = db.by_name.find(key_d(w, d) * 1000 + last);
  return it == db.by_name.end() ? -1 : it->second;
}

// NewOrder (TPC-C 2.4; SURVEY §8(c) procedure table)
void proc_neworder(ProcCtx& x, const uint8_t* p, int64_t* res) {
  uint64_t w = rd<uint16_t>(p, 0), d = p[2], n = p[3], c = rd<uint16_t>(p, 4);
  int64_t w_tax = x.get(TW, w, W_TAX);            // static reads: unmarked
  int64_t d_tax = x.get(TD, key_d(w, d), D_TAX);
  int64_t disc = x.get(TC, key_c(w, d, c), C_DISCOUNT);
  x.get(TC, key_c(w, d, c), C_CREDIT);
  x.get(TC, key_c(w, d, c), C_LAST);
  // fetch-ADD of D_NEXT_O_ID: an ADD unit (R12); the value is assigned at apply
  x.acc(TD, key_d(w, d), x.grp(TD, D_NEXT_O_ID), ACC_A);
  x.tx.is_neworder = true;
  x.tx.no_dkey = key_d(w, d);
  int64_t sum_amount = 0;
  bool all_local = true;
  for (uint64_t l = 0; l < n; ++l) {
    const uint8_t* L = p + 8 + 8 * l;
    uint64_t i = rd<uint32_t>(L, 0), sw = rd<uint16_t>(L, 4), qty = L[6];
    if (!x.exists(TI, i)) { x.tx.user_abort = true; continue; }  // rollback (R11)
    int64_t price = x.get(TI, i, I_PRICE);
    uint64_t sk = key_s(sw, i);
    int64_t q = x.get(TS, sk, S_QUANTITY);
    int64_t nq = q >= int64_t(qty) + 10 ? q - int64_t(qty) : q - int64_t(qty) + 91;
    x.acc(TS, sk, x.grp(TS, S_QUANTITY), ACC_W);
    x.set(TS, sk, S_QUANTITY, nq);
    x.upd_add(TS, sk, S_YTD, int64_t(qty));
    x.upd_add(TS, sk, S_ORDER_CNT, 1);
    x.upd_add(TS, sk, S_REMOTE_CNT, sw != w ? 1 : 0);
    if (sw != w) all_local = false;
    int64_t amount = int64_t(qty) * price;
    sum_amount += amount;
    x.tx.ol_vals.push_back({int64_t(i), int64_t(sw), int64_t(qty), amount, 0});
  }
  x.tx.o_vals = {int64_t(c), x.clock, int64_t(n), all_local ? 1 : 0, 0};
  res[0] = 0;  // o_id: assigned at apply if committed
  res[1] = sum_amount * (10000 - disc) * (10000 + w_tax + d_tax) / 100000000;
  res[2] = sum_amount;
  res[3] = 0;
}

// Payment (TPC-C 2.5)
void proc_payment(ProcCtx& x, const uint8_t* p, int64_t* res) {
  uint64_t w = rd<uint16_t>(p, 0), d = p[2], by_name = p[3], cw = rd<uint16_t>(p, 4), cd = p[6];
  uint64_t cid = rd<uint16_t>(p, 8), clast = rd<uint16_t>(p, 10);
  int64_t amount = rd<int64_t>(p, 16);
  if (by_name) {
    int64_t c = lookup_by_name(x.db, cw, cd, clast);
    if (c < 0) { x.ok = false; return; }
    cid = uint64_t(c);
  }
  uint64_t ck = key_c(cw, cd, cid);
  x.upd_add(TW, w, W_YTD, amount);
  x.upd_add(TD, key_d(w, d), D_YTD, amount);
  bool delayed = x.add_col(TC, C_BALANCE);
  res[0] = int64_t(cid);
  res[1] = delayed ? 0 : x.get(TC, ck, C_BALANCE);  // pre-image (strict only)
  res[2] = 0;
  res[3] = 0;
  x.upd_add(TC, ck, C_BALANCE, -amount);
  x.upd_add(TC, ck, C_YTD_PAYMENT, amount);
  x.upd_add(TC, ck, C_PAYMENT_CNT, 1);
  // HISTORY: keyless append, no marks
  x.tx.eff.push_back({E_APPEND, TH, 0, 0, 0,
                      {int64_t(cid), int64_t(cd), int64_t(cw), int64_t(d), int64_t(w), x.clock, amount,
                       int64_t(x.tid), 0}});
}

// OrderStatus (TPC-C 2.6) with a predefined order key
void proc_orderstatus(ProcCtx& x, const uint8_t* p, int64_t* res) {
  uint64_t w = rd<uint16_t>(p, 0), d = p[2], by_name = p[3], cid = rd<uint16_t>(p, 4), clast = rd<uint16_t>(p, 6);
  if (by_name) {
    int64_t c = lookup_by_name(x.db, w, d, clast);
    if (c < 0) { x.ok = false; return; }
    cid = uint64_t(c);
  }
  uint64_t ck = key_c(w, d, cid);
  int64_t bal = x.get(TC, ck, C_BALANCE);
  x.rd_mark(TC, ck, C_BALANCE);
  uint64_t o = uint64_t(x.get(TC, ck, C_INIT_O_ID));
  uint64_t ok = key_o(w, d, o);
  int64_t carrier = x.get(TO, ok, O_CARRIER_ID);
  x.rd_mark(TO, ok, O_CARRIER_ID);
  int64_t cnt = x.get(TO, ok, O_OL_CNT);
  int64_t sum_dd = 0;
  for (int64_t l = 1; l <= cnt; ++l) {
    uint64_t lk = key_ol(w, d, o, uint64_t(l));
    sum_dd += x.get(TOL, lk, OL_DELIVERY_D);
    x.rd_mark(TOL, lk, OL_DELIVERY_D);
  }
  res[0] = int64_t(cid);
  res[1] = bal;
  res[2] = carrier;
  res[3] = sum_dd;
}

// Delivery (TPC-C 2.7), cursor column D_NEXT_DELIV_O_ID (R14)
void proc_delivery(ProcCtx& x, const uint8_t* p, int64_t* res) {
  uint64_t w = rd<uint16_t>(p, 0);
  int64_t carrier = p[2];
  int64_t delivered = 0, total = 0;
  for (uint64_t d = 1; d <= 10; ++d) {
    uint64_t dk = key_d(w, d);
    int64_t o = x.get(TD, dk, D_NEXT_DELIV_O_ID);
    x.acc(TD, dk, x.grp(TD, D_NEXT_DELIV_O_ID), ACC_W);  // RMW of the cursor
    uint64_t nok = key_o(w, d, uint64_t(o));
    if (!x.exists(TNO, nok)) {
      // queue empty in S: READ the D_NEXT_O_ID unit (conflicts with same-batch NewOrders)
      x.acc(TD, dk, x.grp(TD, D_NEXT_O_ID), ACC_R);
      x.set(TD, dk, D_NEXT_DELIV_O_ID, o);
      continue;
    }
    x.set(TD, dk, D_NEXT_DELIV_O_ID, o + 1);
    for (uint32_t g = 0; g < x.db.tables[TNO].n_groups; ++g) x.acc(TNO, nok, g, ACC_W);
    x.tx.eff.push_back({E_DELETE, TNO, nok, 0, 0, {}});
    x.acc(TO, nok, x.grp(TO, O_CARRIER_ID), ACC_W);
    x.set(TO, nok, O_CARRIER_ID, carrier);
    uint64_t cid = uint64_t(x.get(TO, nok, O_C_ID));
    int64_t cnt = x.get(TO, nok, O_OL_CNT);
    int64_t sum = 0;
    for (int64_t l = 1; l <= cnt; ++l) {
      uint64_t lk = key_ol(w, d, uint64_t(o), uint64_t(l));
      x.acc(TOL, lk, x.grp(TOL, OL_DELIVERY_D), ACC_W);
      x.set(TOL, lk, OL_DELIVERY_D, x.clock);
      sum += x.get(TOL, lk, OL_AMOUNT);
    }
    uint64_t ck = key_c(w, d, cid);
    x.upd_add(TC, ck, C_BALANCE, sum);
    x.upd_add(TC, ck, C_DELIVERY_CNT, 1);
    ++delivered;
    total += sum;
  }
  res[0] = delivered;
  res[1] = total;
  res[2] = 0;
  res[3] = 0;
}

// StockLevel (TPC-C 2.8): window [nx-20, nx) derived from D_NEXT_O_ID (R14)
void proc_stocklevel(ProcCtx& x, const uint8_t* p, int64_t* res) {
  uint64_t w = rd<uint16_t>(p, 0), d = p[2];
  int64_t thr = p[3];
  uint64_t dk = key_d(w, d);
  int64_t nx = x.get(TD, dk, D_NEXT_O_ID);
  x.rd_mark(TD, dk, D_NEXT_O_ID);
  std::vector<int64_t> items;
  for (int64_t o = nx - 20; o < nx; ++o) {
    uint64_t ok = key_o(w, d, uint64_t(o));
    int64_t cnt = x.get(TO, ok, O_OL_CNT);
    for (int64_t l = 1; l <= cnt; ++l) items.push_back(x.get(TOL, key_ol(w, d, uint64_t(o), uint64_t(l)), OL_I_ID));
  }
  std::sort(items.begin(), items.end());
  items.erase(std::unique(items.begin(), items.end()), items.end());
  int64_t low = 0;
  for (int64_t i : items) {
    uint64_t sk = key_s(w, uint64_t(i));
    if (x.get(TS, sk, S_QUANTITY) < thr) ++low;
    x.rd_mark(TS, sk, S_QUANTITY);
  }
  res[0] = low;
  res[1] = nx;
  res[2] = 0;
  res[3] = 0;
}

int validate_proc(const Db& db, uint32_t n, const uint64_t* tid, const uint8_t* type, const uint8_t* params) {
  const uint64_t W = db.n_warehouses;
  for (uint32_t r = 1; r < n; ++r)
    if (tid[r] <= tid[r - 1]) return ORC_EINVAL;
  auto okw = [&](uint64_t w) { return w >= 1 && w <= W; };
  auto okd = [](uint64_t d) { return d >= 1 && d <= 10; };
  for (uint32_t r = 0; r < n; ++r) {
    const uint8_t* p = params + 128ull * r;
    uint64_t w = rd<uint16_t>(p, 0);
    if (!okw(w)) return ORC_EINVAL;
    switch (type[r]) {
      case P_NEWORDER: {
        uint64_t nl = p[3], c = rd<uint16_t>(p, 4);
        if (!okd(p[2]) || nl < 1 || nl > 15 || c < 1 || c > 3000) return ORC_EINVAL;
        for (uint64_t l = 0; l < nl; ++l) {
          const uint8_t* L = p + 8 + 8 * l;
          uint64_t i = rd<uint32_t>(L, 0);
          if (!okw(rd<uint16_t>(L, 4)) || L[6] < 1 || L[6] > 10 || i < 1 || i > 100001) return ORC_EINVAL;
          for (uint64_t m = 0; m < l; ++m)
            if (rd<uint32_t>(p + 8 + 8 * m, 0) == i) return ORC_EINVAL;  // R10
        }
        break;
      }
      case P_PAYMENT:
        if (!okd(p[2]) || !okw(rd<uint16_t>(p, 4)) || !okd(p[6]) || p[3] > 1) return ORC_EINVAL;
        if (p[3] ? rd<uint16_t>(p, 10) > 999 : (rd<uint16_t>(p, 8) < 1 || rd<uint16_t>(p, 8) > 3000)) return ORC_EINVAL;
        break;
      case P_ORDERSTATUS:
        if (!okd(p[2]) || p[3] > 1) return ORC_EINVAL;
        if (p[3] ? rd<uint16_t>(p, 6) > 999 : (rd<uint16_t>(p, 4) < 1 || rd<uint16_t>(p, 4) > 3000)) return ORC_EINVAL;
        break;
      case P_DELIVERY:
        if (p[2] < 1 || p[2] > 10) return ORC_EINVAL;
        break;
      case P_STOCKLEVEL:
        if (!okd(p[2])) return ORC_EINVAL;
        break;
      default:
        return ORC_EINVAL;
    }
  }
  return ORC_OK;
}

void build_by_name(Db& db) {
  // P:297 secondary index; TPC-C 2.5.2.2: customers with C_LAST sorted by C_FIRST,
  // take position ceil(n/2) (1-based); ties on C_FIRST broken by c_id.
  db.by_name.clear();
  const Table& C = db.tables[TC];
  std::map<uint64_t, std::vector<std::pair<int64_t, int64_t>>> groups;
  for (uint64_t r = 0; r < C.rows(); ++r) {
    if (!C.valid[r]) continue;
    uint64_t k = C.key[r];
    uint64_t dk = (k - 1) / 3000, c = (k - 1) % 3000 + 1;
    groups[dk * 1000 + uint64_t(C.col[C_LAST][r])].push_back({C.col[C_FIRST][r], int64_t(c)});
  }
  for (auto& kv : groups) {
    auto& v = kv.second;
    std::sort(v.begin(), v.end());
    size_t pos = (v.size() + 1) / 2;  // ceil(n/2), 1-based
    db.by_name[kv.first] = v[pos - 1].second;
  }
  db.by_name_built = true;
}

}  // namespace

// ---------------------------------------------------------------------------
// C ABI (ctypes, tests only)
// ---------------------------------------------------------------------------
extern "C" {

void* orc_create(uint32_t n_tables, uint32_t n_warehouses) {
  Db* db = new Db();
  db->tables.resize(n_tables);
  db->n_warehouses = n_warehouses;
  return db;
}

void orc_destroy(void* h) { delete static_cast<Db*>(h); }

// NEXT-1: logical reordering (commit rule WAW or (RAW and WAR) aborts)
void orc_set_reorder(void* h, int on) { static_cast<Db*>(h)->reorder = on != 0; }

// SURVEY §8(d) secondary baseline: O1-O3 on `threads` std::threads (1 = the plain oracle)
void orc_set_threads(void* h, uint32_t threads) { static_cast<Db*>(h)->threads = threads ? threads : 1; }

int orc_define_table(void* h, uint32_t t, uint32_t n_cols, const uint8_t* group, const uint8_t* is_add,
                     uint32_t n_groups, uint32_t has_pk) {
  Db& db = *static_cast<Db*>(h);
  if (t >= db.tables.size()) return ORC_EINVAL;
  Table& T = db.tables[t];
  T = Table();
  T.defined = true;
  T.n_cols = n_cols;
  T.n_groups = n_groups;
  T.has_pk = has_pk != 0;
  T.group.assign(group, group + n_cols);
  T.is_add.assign(is_add, is_add + n_cols);
  T.col.assign(n_cols, {});
  for (uint32_t c = 0; c < n_cols; ++c) {
    if (T.group[c] != STATIC_GROUP && T.group[c] >= n_groups) return ORC_EINVAL;
    if (T.is_add[c] && T.group[c] == STATIC_GROUP) return ORC_EINVAL;
  }
  // an ADD group holds ADD columns only (reading R7b)
  for (uint32_t c = 0; c < n_cols; ++c)
    for (uint32_t e = 0; e < n_cols; ++e)
      if (T.group[c] != STATIC_GROUP && T.group[c] == T.group[e] && T.is_add[c] != T.is_add[e]) return ORC_EINVAL;
  return ORC_OK;
}

int orc_load_table(void* h, uint32_t t, uint64_t n_rows, const uint64_t* keys, const int64_t* cols) {
  Db& db = *static_cast<Db*>(h);
  if (t >= db.tables.size() || !db.tables[t].defined) return ORC_EINVAL;
  Table& T = db.tables[t];
  std::vector<int64_t> vals(T.n_cols);
  for (uint64_t r = 0; r < n_rows; ++r) {
    for (uint32_t c = 0; c < T.n_cols; ++c) vals[c] = cols[c * n_rows + r];
    uint64_t k = T.has_pk ? keys[r] : 0;
    if (T.has_pk && (k == KEY_RESERVED || T.pk.count(k))) return ORC_EINVAL;
    T.append(k, vals);
  }
  if (t == TC) db.by_name_built = false;
  return ORC_OK;
}

// One OPS batch.  status[n], reads[n_ops].
int orc_run_ops(void* h, uint32_t n, const uint64_t* tid, const uint32_t* op_begin, const void* ops_v,
                const int64_t* args, uint8_t* status, int64_t* reads) {
  Db& db = *static_cast<Db*>(h);
  const uint8_t* ops = static_cast<const uint8_t*>(ops_v);
  int rc = validate_ops(db, n, tid, op_begin, ops);
  if (rc) return rc;
  std::vector<TxnExec> ex(n);
  parallel_ranges(n, db.threads, [&](uint32_t lo, uint32_t hi) {
    for (uint32_t r = lo; r < hi; ++r)  // O1 (rank order irrelevant: all reads hit S)
      for (uint32_t i = op_begin[r]; i < op_begin[r + 1]; ++i)
        exec_op(db, read_op(ops + 16ull * i), args[i], ex[r], &reads[i]);
  });
  std::vector<uint8_t> st;
  if (db.threads > 1) decide_threads(ex, st, db.reorder, db.threads);
  else decide(ex, st, db.reorder);  // O2 + O3
  for (uint32_t r = 0; r < n; ++r) {  // O4 in TID order
    status[r] = st[r];
    if (st[r] != ST_COMMIT) continue;
    for (const Effect& e : ex[r].eff)
      if (apply_effect(db, e)) return ORC_EINTERNAL;
  }
  return ORC_OK;
}

// One TPC-C PROC batch.  status[n], results[4n].
int orc_run_tpcc(void* h, uint32_t n, const uint64_t* tid, const uint8_t* type, const void* params_v,
                 int64_t clock, uint8_t* status, int64_t* results) {
  Db& db = *static_cast<Db*>(h);
  const uint8_t* params = static_cast<const uint8_t*>(params_v);
  int rc = validate_proc(db, n, tid, type, params);
  if (rc) return rc;
  if (!db.by_name_built) build_by_name(db);
  std::vector<TxnExec> ex(n);
  std::vector<uint8_t> bad(n, 0);
  parallel_ranges(n, db.threads, [&](uint32_t lo, uint32_t hi) {
    for (uint32_t r = lo; r < hi; ++r) {  // O1
      ProcCtx x{db, ex[r], clock, tid[r]};
      const uint8_t* p = params + 128ull * r;
      int64_t* res = results + 4ull * r;
      switch (type[r]) {
        case P_NEWORDER: proc_neworder(x, p, res); break;
        case P_PAYMENT: proc_payment(x, p, res); break;
        case P_ORDERSTATUS: proc_orderstatus(x, p, res); break;
        case P_DELIVERY: proc_delivery(x, p, res); break;
        case P_STOCKLEVEL: proc_stocklevel(x, p, res); break;
      }
      bad[r] = !x.ok;
    }
  });
  for (uint32_t r = 0; r < n; ++r)
    if (bad[r]) return ORC_EINTERNAL;
  std::vector<uint8_t> st;
  if (db.threads > 1) decide_threads(ex, st, db.reorder, db.threads);
  else decide(ex, st, db.reorder);  // O2 + O3
  for (uint32_t r = 0; r < n; ++r) {  // O4: committed write sets (a unit has at most one plain
    status[r] = st[r];               // writer; adds commute; fetch pre-images in TID order)
    if (st[r] != ST_COMMIT) continue;
    for (const Effect& e : ex[r].eff)
      if (apply_effect(db, e)) return ORC_EINTERNAL;
    if (ex[r].is_neworder) {
      // fetch pre-image of D_NEXT_O_ID in TID order (P:241 prefix sum; R12)
      Table& D = db.tables[TD];
      uint64_t drow;
      if (!D.find(ex[r].no_dkey, &drow)) return ORC_EINTERNAL;
      int64_t o = D.col[D_NEXT_O_ID][drow];
      D.col[D_NEXT_O_ID][drow] = o + 1;
      results[4ull * r] = o;
      uint64_t dk = ex[r].no_dkey;
      uint64_t okey = (dk << 32) | uint64_t(o);
      if (apply_effect(db, {E_INSERT, TO, okey, 0, 0, ex[r].o_vals})) return ORC_EINTERNAL;
      if (apply_effect(db, {E_INSERT, TNO, okey, 0, 0, {o}})) return ORC_EINTERNAL;
      for (size_t l = 0; l < ex[r].ol_vals.size(); ++l)
        if (apply_effect(db, {E_INSERT, TOL, okey * 16 + (l + 1), 0, 0, ex[r].ol_vals[l]})) return ORC_EINTERNAL;
    }
  }
  return ORC_OK;
}

uint64_t orc_count_rows(void* h, uint32_t t) {
  const Table& T = static_cast<Db*>(h)->tables[t];
  uint64_t n = 0;
  for (uint8_t v : T.valid) n += v;
  return n;
}

uint32_t orc_n_cols(void* h, uint32_t t) { return static_cast<Db*>(h)->tables[t].n_cols; }

// Canonical dump (O5): keyed tables sorted by key; keyless tables sorted by the
// full column tuple.  keys[n] (keyed only), cols[n_cols * n] col-major.
int orc_dump_table(void* h, uint32_t t, uint64_t* keys, int64_t* cols) {
  const Table& T = static_cast<Db*>(h)->tables[t];
  std::vector<uint64_t> rows;
  for (uint64_t r = 0; r < T.rows(); ++r)
    if (T.valid[r]) rows.push_back(r);
  if (T.has_pk) {
    std::sort(rows.begin(), rows.end(), [&](uint64_t a, uint64_t b) { return T.key[a] < T.key[b]; });
  } else {
    std::sort(rows.begin(), rows.end(), [&](uint64_t a, uint64_t b) {
      for (uint32_t c = 0; c < T.n_cols; ++c)
        if (T.col[c][a] != T.col[c][b]) return T.col[c][a] < T.col[c][b];
      return false;
    });
  }
  const uint64_t n = rows.size();
  for (uint64_t i = 0; i < n; ++i) {
    if (T.has_pk && keys) keys[i] = T.key[rows[i]];
    for (uint32_t c = 0; c < T.n_cols; ++c) cols[c * n + i] = T.col[c][rows[i]];
  }
  return ORC_OK;
}

}  // extern "C"
