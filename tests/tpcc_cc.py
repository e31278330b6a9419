"""TPC-C consistency conditions (TPC-C spec clause 3.3.2, cited by PAPER.md as [1])
evaluated on canonical table dumps -- used on oracle output and on GPU output.

dumps: table_id -> (keys u64[n] | None, cols int64[n_cols, n]).
Returns a dict name -> bool.
"""
import numpy as np
import pandas as pd

from workloads.formats import (T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_HISTORY, T_NEW_ORDER,
                               T_ORDER, T_ORDER_LINE, T_STOCK, TPCC_COLS)


def _df(dumps, t):
    keys, cols = dumps[t]
    d = pd.DataFrame({name: cols[i] for i, name in enumerate(TPCC_COLS[t])})
    if keys is not None:
        d["key"] = keys.astype(np.uint64)
    return d


def check(dumps, first_new_o=3001):
    W = _df(dumps, T_WAREHOUSE)
    D = _df(dumps, T_DISTRICT)
    C = _df(dumps, T_CUSTOMER)
    H = _df(dumps, T_HISTORY)
    NO = _df(dumps, T_NEW_ORDER)
    O = _df(dumps, T_ORDER)
    OL = _df(dumps, T_ORDER_LINE)
    S = _df(dumps, T_STOCK)
    out = {}
    W["w"] = W["key"].astype(np.int64)
    D["w"] = (D["key"].astype(np.int64) - 1) // 10
    D["d"] = (D["key"].astype(np.int64) - 1) % 10 + 1
    D["dk"] = D["key"].astype(np.int64)
    C["dk"] = (C["key"].astype(np.int64) - 1) // 3000
    C["c"] = (C["key"].astype(np.int64) - 1) % 3000 + 1
    for df in (NO, O):
        df["dk"] = (df["key"] >> np.uint64(32)).astype(np.int64)
        df["o"] = (df["key"] & np.uint64(0xFFFFFFFF)).astype(np.int64)
    OL["okey"] = OL["key"] >> np.uint64(4)
    OL["dk"] = (OL["okey"] >> np.uint64(32)).astype(np.int64)
    OL["o"] = (OL["okey"] & np.uint64(0xFFFFFFFF)).astype(np.int64)
    H["dk"] = H["H_W_ID"] * 10 + H["H_D_ID"]
    H["cdk"] = H["H_C_W_ID"] * 10 + H["H_C_D_ID"]

    # CC1: W_YTD = sum(D_YTD)
    s = D.groupby("w")["D_YTD"].sum()
    out["CC1"] = bool((W.set_index("w")["W_YTD"] == s.reindex(W["w"]).values).all())
    # CC2: D_NEXT_O_ID - 1 = max(O_ID) = max(NO_O_ID)
    mo = O.groupby("dk")["o"].max().reindex(D["dk"]).values
    mno = NO.groupby("dk")["o"].max().reindex(D["dk"]).values
    ok = (D["D_NEXT_O_ID"].values - 1 == mo)
    ok &= np.isnan(mno) | (D["D_NEXT_O_ID"].values - 1 == mno)
    out["CC2"] = bool(ok.all())
    # CC3: max(NO_O_ID) - min(NO_O_ID) + 1 = count(NEW_ORDER) per district
    g = NO.groupby("dk")["o"]
    out["CC3"] = bool(((g.max() - g.min() + 1) == g.count()).all())
    # CC4: sum(O_OL_CNT) = count(ORDER_LINE) per district
    out["CC4"] = bool((O.groupby("dk")["O_OL_CNT"].sum().sort_index() ==
                       OL.groupby("dk").size().reindex(O.groupby("dk").size().index).sort_index()).all())
    # CC5: O_CARRIER_ID = 0 iff a NEW_ORDER row exists
    has_no = O["key"].isin(NO["key"])
    out["CC5"] = bool(((O["O_CARRIER_ID"] == 0) == has_no).all())
    # CC6: O_OL_CNT = number of ORDER_LINE rows of the order
    cnt = OL.groupby("okey").size()
    out["CC6"] = bool((O["O_OL_CNT"].values == cnt.reindex(O["key"].values).fillna(0).values).all())
    # CC7: OL_DELIVERY_D = 0 iff O_CARRIER_ID = 0
    car = O.set_index("key")["O_CARRIER_ID"].reindex(OL["okey"].values).values
    out["CC7"] = bool(((OL["OL_DELIVERY_D"].values == 0) == (car == 0)).all())
    # CC8: W_YTD = sum(H_AMOUNT) per warehouse
    hw = H.groupby("H_W_ID")["H_AMOUNT"].sum()
    out["CC8"] = bool((W.set_index("w")["W_YTD"] == hw.reindex(W["w"]).values).all())
    # CC9: D_YTD = sum(H_AMOUNT) per district
    hd = H.groupby("dk")["H_AMOUNT"].sum()
    out["CC9"] = bool((D["D_YTD"].values == hd.reindex(D["dk"]).values).all())
    # CC10: C_BALANCE = sum(delivered OL_AMOUNT) - sum(H_AMOUNT) per customer
    OLd = OL[OL["OL_DELIVERY_D"] != 0]
    cust_of_order = O.set_index("key")["O_C_ID"]
    OLd = OLd.assign(c=cust_of_order.reindex(OLd["okey"].values).values)
    dsum = OLd.groupby(["dk", "c"])["OL_AMOUNT"].sum()
    hsum = H.groupby(["cdk", "H_C_ID"])["H_AMOUNT"].sum()
    idx = pd.MultiIndex.from_arrays([C["dk"], C["c"]])
    dv = dsum.reindex(idx).fillna(0).values
    hv = hsum.reindex(idx).fillna(0).values
    out["CC10"] = bool((C["C_BALANCE"].values == dv - hv).all())
    # CC12: C_BALANCE + C_YTD_PAYMENT = sum(delivered OL_AMOUNT)
    out["CC12"] = bool((C["C_BALANCE"].values + C["C_YTD_PAYMENT"].values == dv).all())
    # extra: C_PAYMENT_CNT = number of HISTORY rows of the customer
    hc = H.groupby(["cdk", "H_C_ID"]).size().reindex(idx).fillna(0).values
    out["PAYCNT"] = bool((C["C_PAYMENT_CNT"].values == hc).all())
    # extra: Delivery cursor = min(NO_O_ID), or D_NEXT_O_ID when the queue is empty
    mnno = NO.groupby("dk")["o"].min().reindex(D["dk"]).values
    exp = np.where(np.isnan(mnno), D["D_NEXT_O_ID"].values, mnno)
    out["CURSOR"] = bool((D["D_NEXT_DELIV_O_ID"].values == exp).all())
    # extra: stock counters = sums over ORDER_LINE rows created by NewOrder (o >= first_new_o)
    OLn = OL[OL["o"] >= first_new_o]
    ow = (OLn["dk"] - 1) // 10
    sk = OLn["OL_SUPPLY_W_ID"] * 100000 + OLn["OL_I_ID"]
    agg = pd.DataFrame({"sk": sk.values, "q": OLn["OL_QUANTITY"].values,
                        "r": (OLn["OL_SUPPLY_W_ID"].values != ow.values).astype(np.int64)}).groupby("sk")
    sidx = S["key"].astype(np.int64).values
    out["S_YTD"] = bool((S["S_YTD"].values == agg["q"].sum().reindex(sidx).fillna(0).values).all())
    out["S_ORDER_CNT"] = bool((S["S_ORDER_CNT"].values == agg.size().reindex(sidx).fillna(0).values).all())
    out["S_REMOTE_CNT"] = bool((S["S_REMOTE_CNT"].values == agg["r"].sum().reindex(sidx).fillna(0).values).all())
    return out
