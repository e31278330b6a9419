"""Input formats shared by the oracle and the CUDA path (inputs only, no method arithmetic).

These are the byte layouts documented in include/ltpg.h (the C-ABI) and
DESIGN.md §"Boundary".  Both sides parse them independently; this module only
builds numpy arrays in that layout.

OPS mode (YCSB and micro-cases) -- one record per operation, 16 bytes:
    u64 key | u8 kind | u8 table | u16 col | u32 aux
plus one int64 argument per op and a CSR ``op_begin[n_txns+1]`` (u32).

PROC mode (TPC-C stored procedures, "pre-compiled, stored
procedures ... A client interacts with the system by setting different
parameters") -- one u8 type and one 128-byte parameter block per txn.
"""
import numpy as np

# ---- OPS mode ---------------------------------------------------------------
OP_DTYPE = np.dtype([("key", "<u8"), ("kind", "u1"), ("table", "u1"),
                     ("col", "<u2"), ("aux", "<u4")])
assert OP_DTYPE.itemsize == 16

SELECT, UPDATE, ADD, INSERT, DELETE, SCAN = 0, 1, 2, 3, 4, 5
KIND_NAMES = ["SELECT", "UPDATE", "ADD", "INSERT", "DELETE", "SCAN"]
COL_COUNT = 0xFFFF          # SCAN column meaning "count present keys"
STATIC = 0xFF               # col_group value of a never-written column
NOT_FOUND = -(1 << 63)      # read result of an absent key (INT64_MIN)
KEY_EMPTY = (1 << 64) - 1   # reserved key value (index sentinel), never a valid key

ST_CONFLICT, ST_COMMIT, ST_USER_ABORT = 0, 1, 2

# ---- PROC mode: TPC-C --------------------------------------------------------
NEW_ORDER, PAYMENT, ORDER_STATUS, DELIVERY, STOCK_LEVEL = 0, 1, 2, 3, 4
PROC_NAMES = ["NewOrder", "Payment", "OrderStatus", "Delivery", "StockLevel"]
PARAM_BYTES = 128
RESULT_SLOTS = 4           # int64 result slots per PROC txn

LINE_DTYPE = np.dtype([("i", "<u4"), ("supply_w", "<u2"), ("qty", "u1"), ("pad", "u1")])
NEWORDER_DTYPE = np.dtype([("w", "<u2"), ("d", "u1"), ("n_lines", "u1"), ("c", "<u2"),
                           ("rbk", "u1"), ("pad", "u1"), ("line", LINE_DTYPE, (15,))])
PAYMENT_DTYPE = np.dtype([("w", "<u2"), ("d", "u1"), ("by_name", "u1"), ("c_w", "<u2"),
                          ("c_d", "u1"), ("pad", "u1"), ("c_id", "<u2"), ("c_last", "<u2"),
                          ("pad2", "<u4"), ("amount", "<i8"), ("rest", "u1", (104,))])
ORDERSTATUS_DTYPE = np.dtype([("w", "<u2"), ("d", "u1"), ("by_name", "u1"), ("c_id", "<u2"),
                              ("c_last", "<u2"), ("rest", "u1", (120,))])
DELIVERY_DTYPE = np.dtype([("w", "<u2"), ("carrier", "u1"), ("pad", "u1"), ("rest", "u1", (124,))])
STOCKLEVEL_DTYPE = np.dtype([("w", "<u2"), ("d", "u1"), ("threshold", "u1"), ("rest", "u1", (124,))])
for _dt in (NEWORDER_DTYPE, PAYMENT_DTYPE, ORDERSTATUS_DTYPE, DELIVERY_DTYPE, STOCKLEVEL_DTYPE):
    assert _dt.itemsize == PARAM_BYTES, _dt

# TPC-C schema (table ids and column order) -- integer-only.
T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_HISTORY, T_NEW_ORDER, T_ORDER, T_ORDER_LINE, T_ITEM, T_STOCK = range(9)
TPCC_TABLE_NAMES = ["WAREHOUSE", "DISTRICT", "CUSTOMER", "HISTORY", "NEW_ORDER", "ORDER",
                    "ORDER_LINE", "ITEM", "STOCK"]
TPCC_COLS = {
    T_WAREHOUSE: ["W_TAX", "W_YTD"],
    T_DISTRICT: ["D_TAX", "D_YTD", "D_NEXT_O_ID", "D_NEXT_DELIV_O_ID"],
    T_CUSTOMER: ["C_DISCOUNT", "C_CREDIT", "C_LAST", "C_FIRST", "C_INIT_O_ID",
                 "C_BALANCE", "C_YTD_PAYMENT", "C_PAYMENT_CNT", "C_DELIVERY_CNT"],
    T_HISTORY: ["H_C_ID", "H_C_D_ID", "H_C_W_ID", "H_D_ID", "H_W_ID", "H_DATE", "H_AMOUNT",
                "H_TID", "H_SEQ"],
    T_NEW_ORDER: ["NO_O_ID"],
    T_ORDER: ["O_C_ID", "O_ENTRY_D", "O_OL_CNT", "O_ALL_LOCAL", "O_CARRIER_ID"],
    T_ORDER_LINE: ["OL_I_ID", "OL_SUPPLY_W_ID", "OL_QUANTITY", "OL_AMOUNT", "OL_DELIVERY_D"],
    T_ITEM: ["I_PRICE", "I_IM_ID"],
    T_STOCK: ["S_QUANTITY", "S_YTD", "S_ORDER_CNT", "S_REMOTE_CNT"],
}
S = STATIC
# Column groups (conflict units = (table,row,group)) and ADD flags.
# strict: every mutable group is a WRITE unit except D_NEXT_O_ID (fetch-ADD, R12).
# delayed: hot attributes become blind ADD units (P:241 delayed update).
TPCC_GROUPS = {
    "strict": {
        T_WAREHOUSE: ([S, 0], [0, 0], 1),
        T_DISTRICT: ([S, 0, 1, 2], [0, 0, 1, 0], 3),
        T_CUSTOMER: ([S, S, S, S, S, 0, 0, 0, 0], [0] * 9, 1),
        T_HISTORY: ([S] * 9, [0] * 9, 0),
        T_NEW_ORDER: ([0], [0], 1),
        T_ORDER: ([S, S, S, S, 0], [0] * 5, 1),
        T_ORDER_LINE: ([S, S, S, S, 0], [0] * 5, 1),
        T_ITEM: ([S, S], [0, 0], 0),
        T_STOCK: ([0, 0, 0, 0], [0, 0, 0, 0], 1),
    },
    "delayed": {
        T_WAREHOUSE: ([S, 0], [0, 1], 1),
        T_DISTRICT: ([S, 0, 1, 2], [0, 1, 1, 0], 3),
        T_CUSTOMER: ([S, S, S, S, S, 0, 0, 0, 0], [0, 0, 0, 0, 0, 1, 1, 1, 1], 1),
        T_HISTORY: ([S] * 9, [0] * 9, 0),
        T_NEW_ORDER: ([0], [0], 1),
        T_ORDER: ([S, S, S, S, 0], [0] * 5, 1),
        T_ORDER_LINE: ([S, S, S, S, 0], [0] * 5, 1),
        T_ITEM: ([S, S], [0, 0], 0),
        T_STOCK: ([0, 1, 1, 1], [0, 1, 1, 1], 2),
    },
}
TPCC_HAS_PK = {t: (t != T_HISTORY) for t in range(9)}


def tpcc_col(table, name):
    return TPCC_COLS[table].index(name)


def pack_ops(keys, kinds, tables, cols, aux=None):
    """Build a structured OP_DTYPE array from column arrays."""
    n = len(keys)
    ops = np.zeros(n, dtype=OP_DTYPE)
    ops["key"] = keys
    ops["kind"] = kinds
    ops["table"] = tables
    ops["col"] = cols
    if aux is not None:
        ops["aux"] = aux
    return ops
