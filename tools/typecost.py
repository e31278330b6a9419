import sys, time, numpy as np, torch
sys.path.insert(0, "/root/repo")
import paper_conf_icde_wei0l0lzj024_b200 as L
from workloads import tpcc
B = 1 << 20
wl0 = tpcc.TpccWorkload(64, seed=0x17C3, mode="strict", mix=tpcc.MIX_FULL)
tables = wl0.initial_tables()
for mix in [(1,0,0,0,0),(0,1,0,0,0),(0,0,1,0,0),(0,0,0,1,0),(0,0,0,0,1),tpcc.MIX_FULL]:
    wl = tpcc.TpccWorkload(64, seed=0x17C3, mode="strict", mix=mix)
    db = L.tpcc_database(wl, max_txns=B, tables=tables, append_batches=3)
    b = wl.batch(B, 1, 0)
    dev = {k: torch.from_numpy(np.ascontiguousarray(v)).cuda() for k, v in b.items()}
    outs = []
    for i in range(4):
        o = db.run_tpcc(dev, 2 + i, stats=True, n_txns=B)
        outs.append(o["stats"])
    st = outs[-1]
    print(mix, {k: round(v, 3) for k, v in st.items() if k.startswith("ms_")}, st["n_commit"], flush=True)
    del db
