#!/usr/bin/env python
"""bench.py -- LTPG per-batch DOCC pipeline on B200 (one JSON line on rank 0).

A "step" is one batch through the whole hot path:
validate + warp division -> claim -> execute + marks -> conflict detection ->
write-back -> commit bitmask / abort list.  Workloads are BASELINE.json configs
(synthetic, seeded).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl ours|reference]

value      committed txns/s, inputs resident in HBM (CUDA events per step, L2
           flushed between steps outside the timed events), max over ranks
e2e        same metric through the public API with pinned HOST inputs/outputs
           (H2D + kernels + D2H inside each timed step)
roofline   dominant kernel: algorithmic bytes / its CUDA-event duration vs the
           measured HBM copy peak (MEASURED_PEAKS.json)
cpu_baseline  the CPU oracle (oracle/) as it stands, 1 thread, on a bounded sample
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "committed txns/sec"
UNIT = "txn/s"

WORKLOADS = {
    # BASELINE.json configs[i]; seed = 0x17C0 + i
    "ycsb_c1": dict(kind="ycsb", cfg=0, n_rows=10_000, theta=0.5, ops=4, batch=1024),
    "tpcc_c2": dict(kind="tpcc", cfg=1, W=1, mix="no_pay", batch=16384, mode="strict"),
    "ycsb_c3": dict(kind="ycsb", cfg=2, n_rows=10_000_000, theta=0.99, ops=10, batch=1 << 20),
    "tpcc_c4": dict(kind="tpcc", cfg=3, W=64, mix="full", batch=1 << 20, mode="strict"),
    "tpcc_c5": dict(kind="tpcc", cfg=4, W=512, mix="no_pay", batch=1 << 20, mode="strict"),
    "tpcc_c4_delayed": dict(kind="tpcc", cfg=3, W=64, mix="full", batch=1 << 20, mode="delayed"),
    # NEXT-1 "high-contention package": delayed update + logical reordering
    "tpcc_c4_opt": dict(kind="tpcc", cfg=3, W=64, mix="full", batch=1 << 20, mode="delayed", reorder=True),
    "tpcc_c2_opt": dict(kind="tpcc", cfg=1, W=1, mix="no_pay", batch=16384, mode="delayed", reorder=True),
    "tpcc_c2_delayed": dict(kind="tpcc", cfg=1, W=1, mix="no_pay", batch=16384, mode="delayed"),
    "ycsb_c3_4ops": dict(kind="ycsb", cfg=2, n_rows=10_000_000, theta=0.99, ops=4, batch=1 << 20),
    # C3 with sparse u64 keys (splitmix64 of the row number): every op probes the PK hash index
    "ycsb_c3_sparse": dict(kind="ycsb", cfg=2, n_rows=10_000_000, theta=0.99, ops=10, batch=1 << 20, sparse=True),
    # NEXT-4: the paper's YCSB suite: Zipf alpha 2.5, 10 ops, 10^7 rows
    **{"ycsb_%s" % L.lower(): dict(kind="ycsb", cfg=2, n_rows=10_000_000, theta=2.5, ops=10, batch=1 << 16,
                                   letter=L) for L in "ABCDE"},
}
DEFAULT_WORKLOAD = "tpcc_c4"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ---- clocks sampler (B200_PROFILING.md "clocks DURING the timed region") ------------------
class ClockSampler:
    """SM clock + throttle reasons sampled every ~2 ms through NVML (nvidia-smi is the
    fallback) on a background thread; the summary covers the samples taken inside the
    windows bench.py marks as timed (device-resident leg and e2e leg)."""
    SMI_Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    # NVML clocks-event reason bits (nvml.h)
    REASONS = {"sw_power_cap": 0x4, "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20,
               "hw_thermal_slowdown": 0x40}

    def __init__(self, index):
        self.index = index
        self.samples = []   # (t, sm_mhz, reason_bits)
        self.windows = []
        self.max_mhz = None
        self.source = None
        self.stop = threading.Event()
        self.ready = threading.Event()  # set at the first sample (or when sampling gave up)

    def __enter__(self):
        self.t = threading.Thread(target=self._loop, daemon=True)
        self.t.start()
        return self

    def mark(self, t0, t1):
        self.windows.append((t0, t1))

    def _nvml_handle(self):
        import pynvml
        pynvml.nvmlInit()
        try:
            import torch
            uuid = str(torch.cuda.get_device_properties(self.index).uuid)
            return pynvml, pynvml.nvmlDeviceGetHandleByUUID(("GPU-" + uuid) if not uuid.startswith("GPU-") else uuid)
        except Exception:
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.index)

    def _loop(self):
        try:
            nv, h = self._nvml_handle()
            self.max_mhz = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
            self.source = "nvml"
            while not self.stop.is_set():
                sm = float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM))
                try:
                    rb = int(nv.nvmlDeviceGetCurrentClocksEventReasons(h))
                except Exception:
                    rb = int(nv.nvmlDeviceGetCurrentClocksThrottleReasons(h))
                self.samples.append((time.time(), sm, rb))
                self.ready.set()
                self.stop.wait(0.002)
            return
        except Exception:
            pass
        self.source = "nvidia-smi"
        while not self.stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.SMI_Q,
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout
                for ln in out.splitlines():
                    f = [x.strip() for x in ln.split(",")]
                    if len(f) < 9:
                        continue
                    names = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")
                    rb = sum(self.REASONS[n] for n, v in zip(names, f[5:9]) if v.lower() == "active")
                    self.max_mhz = float(f[2])
                    self.samples.append((time.time(), float(f[1]), rb))
                    self.ready.set()
            except Exception:
                pass
            self.stop.wait(0.05)
        self.ready.set()

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(timeout=6)
        self.ready.set()

    def summary(self):
        inside = [x for x in self.samples if any(t0 <= x[0] <= t1 for t0, t1 in self.windows)]
        if not inside:  # timed legs shorter than the sampling period: the samples bracketing them
            for t0, t1 in self.windows:
                before = [x for x in self.samples if x[0] < t0]
                after = [x for x in self.samples if x[0] > t1]
                inside += before[-1:] + after[:1]
        use = inside or self.samples
        reasons = sorted(n for n, bit in self.REASONS.items() if any(x[2] & bit for x in use))
        return {"sm_mhz": statistics.median(x[1] for x in use) if use else None, "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(use), "source": self.source,
                "window": ("samples inside (or, for legs shorter than the sampling period, "
                           "bracketing) the timed legs" if inside else "all samples")}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("hbm_gbs", 6469.3), "measured"
    return 6650.0, "fallback"


def ncu_traffic(workload, kernel_substr):
    """dram read+write bytes per launch of the kernel from the committed `ncu --set full`
    summary of this workload (profiles/ncu_r02_<workload>.json, else the round-1 one), or None."""
    p = next((q for q in (os.path.join(ROOT, "profiles", "ncu_r0%d_%s.json" % (k, workload)) for k in (2, 1))
              if os.path.exists(q)), None)
    if p is None:
        return None
    try:  # summed over every instantiation that matches (the execute stage may be two launches)
        d = json.load(open(p))
        vals = [v.get("dram_bytes") for k, v in d.get("kernels", {}).items()
                if kernel_substr in k and v.get("dram_bytes") is not None]
        return sum(vals) if vals else None
    except Exception:
        return None


# ---- workloads ------------------------------------------------------------------------------
def make_workload(name, rank=0):
    # every rank builds the same global workload (partitioned multi-GPU mode, §8(e))
    w = WORKLOADS[name]
    seed = 0x17C0 + w["cfg"]
    if w["kind"] == "ycsb":
        from workloads.ycsb import YcsbWorkload, ycsb_letter
        if w.get("letter"):
            return ycsb_letter(w["letter"], w["n_rows"], theta=w["theta"], ops_per_txn=w["ops"], seed=seed)
        return YcsbWorkload(w["n_rows"], theta=w["theta"], ops_per_txn=w["ops"], seed=seed,
                            sparse_keys=w.get("sparse", False))
    from workloads import tpcc
    mix = tpcc.MIX_FULL if w["mix"] == "full" else tpcc.MIX_NO_PAY
    return tpcc.TpccWorkload(w["W"], seed=seed, mode=w["mode"], mix=mix)


def open_database(name, wl, n_batches, flags=0, device=0, rank=0, world=1, **kw):
    """The database exactly as the bench times it (also used by the full-size parity tests):
    append regions sized for the worst case of one batch plus the appends of `n_batches`
    batches (every NewOrder / Payment committing; 10.5 lines per NewOrder on average)."""
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    w = WORKLOADS[name]
    B = w["batch"]
    if w.get("reorder"):
        flags |= ltpg.LTPG_FLAG_REORDER
    if w["kind"] == "ycsb":  # inserts (YCSB D/E) of every batch
        return ltpg.ycsb_database(wl, max_txns=B, max_ops=B * w["ops"], flags=flags, device=device,
                                  rank=rank, world=world,
                                  capacity=w["n_rows"] + n_batches * B * w["ops"] // 10 + 1024, **kw)
    from workloads.formats import T_ORDER, T_NEW_ORDER, T_ORDER_LINE, T_HISTORY
    tabs = wl.initial_tables()
    no, pay = B * wl.mix[0], B * wl.mix[1]
    cap = {T_ORDER: no * (1 + n_batches), T_NEW_ORDER: no * (1 + n_batches),
           T_ORDER_LINE: 15 * no + 10.5 * no * n_batches, T_HISTORY: pay * (1 + n_batches)}
    cap = {t: int(tabs[t][1].shape[1] + v) + 1024 for t, v in cap.items()}
    return ltpg.tpcc_database(wl, max_txns=B, tables=tabs, capacity=cap, flags=flags, device=device,
                              rank=rank, world=world, **kw)


def exec_algorithmic_bytes(batch, sparse=False):
    """Algorithmic bytes of the OPS execute kernel: per op 16 B op record +
    32 B data sector + 8 B result + 8 B unit reference = 64 B; + 64 B per marking op
    (UPDATE/ADD/INSERT/DELETE: atomic sector RMW).  Dense key ranges map key -> row by
    arithmetic (identity bucket function), so no index bytes are counted; sparse keys
    add one 32-byte index-slot sector per op (linear probing at load factor <= 1/2)."""
    kinds = batch["ops"]["kind"]
    n = len(kinds)
    marking = int(np.isin(kinds, [1, 2, 3, 4]).sum())
    return 64 * n + 64 * marking + (32 * n if sparse else 0)


def tpcc_exec_algorithmic_bytes(batch, mode):
    """Algorithmic bytes of the TPC-C execute kernel: 128 B parameter block,
    32 B per random column read or index probe of a sparse-keyed table, 64 B per mark (atomic
    sector RMW) outside the per-block shared-memory WAREHOUSE / DISTRICT marks, contiguous order
    lines at element size, 32 B result + 4 B per logged row.
    W/D/C/I/S rows are found by arithmetic (dense keys); ORDER_LINE rows from ORDER.
    Delivery / StockLevel use the expected line counts (10 / 190 distinct items) and are
    counted once per warehouse / district, as they are executed."""
    ty = batch["type"]
    p = batch["params"]
    nl = p[:, 3].astype(np.int64)
    delayed = mode == "delayed"
    by_name = p[:, 3].astype(bool)
    b = np.zeros(len(ty), np.int64)
    no = ty == 0
    # (the WAREHOUSE / DISTRICT marks are aggregated per block in shared memory and flushed once
    # per touched unit and block: not counted per txn)
    b[no] = 128 + 3 * 32 + nl[no] * (32 + 64 * (1 + delayed) + 4) + 32 + 4
    pay = ty == 1
    b[pay] = 128 + 64 + 32 * (not delayed) + 4 * by_name[pay] + 16 + 32
    b[ty == 2] = 128 + 2 * 32 + 32 + 2 * 32 + 4 + 10 * 8 + 32 + 68
    # Delivery is shared per warehouse (only its smallest rank executes): the
    # full cost once per warehouse, a parameter sector per other Delivery
    w = p[:, 0].astype(np.int64) | (p[:, 1].astype(np.int64) << 8)
    dl = ty == 3
    n_dw = len(np.unique(w[dl]))
    b[dl] = 32
    full_dl = 128 + 10 * (32 + 64 + 32 + 32 + 3 * 32 + 4 + 64 + 10 * (8 + 16) + 64) + 32
    # StockLevel is evaluated once per district on the side stream (k_sl_*; inside the timed
    # execute stage): the window scan once per district, claim + result per txn
    sl = ty == 4
    n_sd = len(np.unique(w[sl] * 16 + p[sl, 2].astype(np.int64)))
    b[sl] = 32 + 32
    full_sl = 32 + 20 * (32 + 32 + 4 + 10 * 8) + 190 * 32 + 32
    return int(b.sum()) + n_dw * full_dl + n_sd * full_sl


def tpcc_random_touches(batch):
    """Independent random row/mark touches of the TPC-C execute stage per batch (the TPC-C analogue
    of ops_random_reads): NewOrder 2 per line (item price read, stock mark) + 3 (W / D / C static
    reads; the district mark is in shared memory); Payment 2 (customer row, customer mark) + 1 by
    name; OrderStatus 4 + its ~10 lines; a Delivery leader per warehouse ~10 x (cursor, 2 probes,
    order row, customer row + ~10 lines) = 150; StockLevel once per district ~20 x 3 + ~190 stock
    rows = 250, + 1 per txn.  Many of these hit L2 (items, marks), so the fraction of the DRAM
    random-read ceiling is an upper estimate of how hard the stage drives the memory system."""
    ty = batch["type"]
    p = batch["params"]
    nl = p[:, 3].astype(np.int64)
    w = p[:, 0].astype(np.int64) | (p[:, 1].astype(np.int64) << 8)
    t = np.zeros(len(ty), np.int64)
    t[ty == 0] = 2 * nl[ty == 0] + 3
    t[ty == 1] = 2 + p[ty == 1, 3].astype(np.int64)
    t[ty == 2] = 14
    t[ty == 4] = 1
    n_dw = len(np.unique(w[ty == 3]))
    n_sd = len(np.unique(w[ty == 4] * 16 + p[ty == 4, 2].astype(np.int64)))
    return int(t.sum()) + 150 * n_dw + 250 * n_sd


def fused_algorithmic_bytes(batch, sparse=False):
    """Algorithmic bytes of the fused OPS kernel (validate + warp-local division + execute):
    the execute bytes above + 16 B per txn (TID 8 B, op_begin 4 B, txn_ins 4 B)."""
    return exec_algorithmic_bytes(batch, sparse) + 16 * len(batch["tid"])


# B200 random-access ceiling measured by tools/randbw.cu (profiles/randbw_r01.txt): independent
# random 8-byte reads from a >> L2 array retire at ~48.6 G/s whatever the load flavour or the
# DRAM bytes fetched per access -- a request-rate limit well below the sequential HBM peak.
RANDOM_READ_CEILING_G = 48.6


def ops_random_reads(batch, sparse=False):
    """Independent random row-sized reads the OPS execute does per batch: one column read per
    SELECT / UPDATE (dense key -> row by arithmetic), one mark-filter read per UPDATE / ADD
    (its atomicMin then hits the line in L2), one read per SCANned key; INSERT / DELETE 2;
    sparse keys: + one index-slot read per op."""
    ops = batch["ops"]
    kinds = ops["kind"]
    n = np.bincount(kinds, minlength=6)
    scan_keys = int(ops["aux"][kinds == 5].astype(np.int64).sum())
    return int(n[0] + 2 * n[1] + n[2] + 2 * (n[3] + n[4]) + scan_keys) + (len(kinds) if sparse else 0)


def step_algorithmic_bytes(batch):
    """Whole-step algorithmic bytes (OPS): exec + detect (8 B uref + 32 B mark sector per op)
    + group (16 B op + 8 B list entry) + per-txn status/bits/flags (~10 B)."""
    n = len(batch["ops"])
    return exec_algorithmic_bytes(batch) + n * (40 + 24) + 10 * len(batch["tid"])


# ---- host CPU ---------------------------------------------------------------------------------------
def host_cpu():
    """CPU model and the cores this process may use (report them)."""
    model = None
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    try:
        n = len(os.sched_getaffinity(0))
    except AttributeError:
        n = os.cpu_count() or 1
    return {"model": model, "nproc": n}


def _oracle_db(name, wl, threads):
    import oracle
    w = WORKLOADS[name]
    db = oracle.ycsb_db(wl) if w["kind"] == "ycsb" else oracle.tpcc_db(wl)
    if w.get("reorder"):
        db.set_reorder(True)
    db.set_threads(threads)
    return db


def _oracle_run(db, kind, b, clock):
    t = time.perf_counter()
    rc, st, _ = db.run_ops(b) if kind == "ycsb" else db.run_tpcc(b, clock=clock)
    dt = time.perf_counter() - t
    assert rc == 0
    return int((st == 1).sum()), dt


# ---- reference arm: the CPU oracle ---------------------------------------------------------------
REF_BUDGET_S = 150.0   # timed oracle work of the whole reference run (the run must end in minutes)


def run_reference(args, name):
    """The reference arm is the CPU oracle (oracle/) on the box's host cores, on the same workload
    and metric as our arm: fresh batches of the workload's full size when K of them fit in
    REF_BUDGET_S on nproc threads (the oracle's SURVEY §8(d) threaded mode), else the largest
    power-of-two sample that does.  Warm-up steps are small untimed samples."""
    w = WORKLOADS[name]
    kind = w["kind"]
    wl = make_workload(name, 0)
    cpu = host_cpu()
    threads = args.ref_threads or cpu["nproc"]
    t0 = time.time()
    db = _oracle_db(name, wl, threads)
    log("oracle load %.1fs (%d threads)" % (time.time() - t0, threads))
    tid, clock = 1, 2
    rate = None
    for s in range(args.warmup):  # untimed; the last one estimates the processing rate
        n = min(w["batch"], 1 << 14)
        _, dt = _oracle_run(db, kind, wl.batch(n, tid, 10_000 + s), clock)
        tid, clock = tid + n, clock + 1
        rate = n / max(dt, 1e-6)
    sample = w["batch"]
    if args.ref_sample:
        sample = min(sample, args.ref_sample)
    while sample > 1024 and rate and sample / rate * args.steps > REF_BUDGET_S:
        sample //= 2
    committed, secs = 0, 0.0
    for s in range(args.steps):
        c, dt = _oracle_run(db, kind, wl.batch(sample, tid, 20_000 + s), clock)
        tid, clock = tid + sample, clock + 1
        committed += c
        secs += dt
    v = committed / secs if secs else 0.0
    desc = ("%d fresh %d-txn batches of %s (full batch %d%s), oracle on %d threads"
            % (args.steps, sample, name, w["batch"], "" if sample == w["batch"] else ": sample bounded by the time budget",
               threads))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * secs / max(args.steps, 1),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int64",
            "data": "synthetic",
            "config": dict(config_of(name, batch=sample), parallelism="CPU oracle, %d threads" % threads),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": desc,
                             "cpu_model": cpu["model"], "nproc": cpu["nproc"]},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_of(name, batch=None):
    w = dict(WORKLOADS[name])
    c = {"workload": name, "baseline_config": w.pop("cfg"), "kind": w.pop("kind")}
    c.update(w)
    if batch is not None:
        c["batch"] = batch
    c["l2"] = "inputs+state larger than L2 (126 MB) and L2 flushed (256 MB write) between timed steps"
    return c


def cpu_baseline_child(name):
    """Runs in a child process (python bench.py --cpu-baseline-child NAME), so the GPU arm's
    process never maps the oracle: the oracle as it stands, 1 thread, on the first bench batch
    (the same 2^k-txn batch the GPU times; bounded by the workload's size: ~10-30 s), then the
    SURVEY §8(d) secondary run on nproc threads on a fresh copy of the same database."""
    w = WORKLOADS[name]
    wl = make_workload(name, 0)
    cpu = host_cpu()
    out = {}
    for threads in (1, cpu["nproc"]):
        t0 = time.time()
        db = _oracle_db(name, wl, threads)
        load_s = time.time() - t0
        c = dt = 0
        nb = 0
        while nb == 0 or (dt < 2.0 and nb < 64):  # the bench's batches 0, 1, ... (>= 2 s of work)
            ci, dti = _oracle_run(db, w["kind"], wl.batch(w["batch"], 1 + nb * w["batch"], nb), 2 + nb)
            c, dt, nb = c + ci, dt + dti, nb + 1
        del db
        out[threads] = (c, dt, load_s, nb)
    c, dt, load_s, nb = out[1]
    cn, dtn, _, nbn = out[cpu["nproc"]]
    assert nb != nbn or c == cn, "threaded oracle disagrees with the single-threaded one"
    res = {"value": c / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
           "sample": "the first %d full %d-txn batch(es) of %s, as the bench generates them (oracle load %.1fs "
                     "not timed; %.1fs of batch work)" % (nb, w["batch"], name, load_s, dt),
           "seconds": dt, "cpu_model": cpu["model"], "nproc": cpu["nproc"], "process": "child (bench.py)",
           "threaded": {"value": cn / dtn, "unit": UNIT, "cores": cpu["nproc"], "seconds": dtn,
                        "kind": "oracle, O1-O3 on nproc std::threads (SURVEY §8(d) secondary)"}}
    print(json.dumps(res), flush=True)


def cpu_baseline(name):
    p = subprocess.run([sys.executable, os.path.abspath(__file__), "--cpu-baseline-child", name],
                       capture_output=True, text=True, timeout=600)
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    if p.returncode or not lines:
        return {"error": "cpu baseline child rc=%d: %s" % (p.returncode, p.stderr[-400:])}
    return json.loads(lines[-1])


def relaunch_under_torchrun(args):
    """`bench.py --gpus N` outside torchrun: re-run this command as N ranks (one per GPU, or
    sharing the GPUs there are) under torch.distributed.run on 127.0.0.1."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=%d" % args.gpus,
           "--master-addr=127.0.0.1", "--master-port=%d" % port, os.path.abspath(__file__)] + sys.argv[1:]
    log("relaunching as %d ranks: %s" % (args.gpus, " ".join(cmd)))
    return subprocess.call(cmd)


# ---- our arm -----------------------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default=os.environ.get("LTPG_BENCH_WORKLOAD", DEFAULT_WORKLOAD),
                    choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-sample", type=int, default=0, help="cap the reference arm's batch (0: full)")
    ap.add_argument("--ref-threads", type=int, default=0, help="reference arm oracle threads (0: nproc)")
    ap.add_argument("--cpu-baseline-child", default=None, help=argparse.SUPPRESS)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-closed-loop", action="store_true")
    ap.add_argument("--flags", type=int, default=0)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.cpu_baseline_child:
        cpu_baseline_child(args.cpu_baseline_child)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch_under_torchrun(args))

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    name = args.workload

    if args.impl == "reference":
        if rank == 0:
            run_reference(args, name)
        return

    import torch
    # one rank per GPU; with fewer GPUs than ranks (a functional check on a 1-GPU box) ranks
    # share devices, the library's exchange then runs over CUDA IPC on one device and the
    # bench plumbing uses gloo (NCCL refuses two ranks on one GPU)
    ndev = torch.cuda.device_count()
    shared = world > ndev
    local = local % ndev
    torch.cuda.set_device(local)
    clk = ClockSampler(local)  # samples through load, warm-up, timed and e2e legs
    if not os.environ.get("LTPG_NO_CLOCKS"):
        clk.__enter__()
    dist = None
    if world > 1:
        import torch.distributed as dist
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg

    w = WORKLOADS[name]
    wl = make_workload(name)
    B = w["batch"]
    if w.get("reorder"):
        args.flags |= ltpg.LTPG_FLAG_REORDER
    fused_front = w["kind"] == "ycsb" and not (args.flags & (ltpg.LTPG_FLAG_REORDER | ltpg.LTPG_FLAG_NO_GROUPING
                                                              | ltpg.LTPG_FLAG_UNFUSED))
    # small single-partition batches run a2..a8 as ONE cooperative kernel (csrc k_ops_small /
    # k_tpcc_small; capi.cu picks it by the same rule): the whole batch is the dominant kernel
    single = (world == 1 and B <= 16384 and (w["kind"] == "ycsb" or w["W"] <= 64) and
              not (args.flags & (ltpg.LTPG_FLAG_LARGE_BUCKETS | ltpg.LTPG_FLAG_NO_SINGLE_LAUNCH)) and
              not (w["kind"] == "ycsb" and args.flags & ltpg.LTPG_FLAG_NO_GROUPING))
    t0 = time.time()
    db = open_database(name, wl, args.warmup + 4 * args.steps + 2, flags=args.flags, device=local,
                       rank=rank, world=world)
    log("rank %d: db loaded in %.1fs" % (rank, time.time() - t0))

    # distinct input batches, cycled (inputs only; every step recomputes everything)
    # (small batches: enough distinct batches that the closed-loop leg's fresh-txn pool lasts)
    n_distinct = 2 if B >= (1 << 18) else min(args.steps + 2, 32)
    host_batches, dev_batches, pin_batches = [], [], []
    # multi-rank TPC-C runs SHARDED batches (SURVEY §8(e) host routing, ltpg_route_tpcc): every
    # rank builds the same global batch, routes out its own shard (the txns touching its
    # warehouses) and uploads only that; it counts the commits of the txns it is home of
    sharded = world > 1 and w["kind"] == "tpcc"
    home_masks, shard_sizes = [], []
    tid = 1
    for i in range(n_distinct):
        b = wl.batch(B, tid, i)
        tid += B
        if sharded:
            b = ltpg.route_tpcc(b, wl.W, world, rank)
            p = b["params"]
            home_masks.append(ltpg.part_of_w(p[:, 0].astype(np.int64) | (p[:, 1].astype(np.int64) << 8),
                                             wl.W, world) == rank)
        shard_sizes.append(len(b["tid"]))
        host_batches.append(b)
    dev = torch.device("cuda", local)

    def to_t(a, pin):
        if not isinstance(a, np.ndarray):
            return a  # scalars (n_global)
        t = torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).copy())
        return t.pin_memory() if pin else t.to(dev)

    home_dev = [torch.from_numpy(m).to(dev) for m in home_masks]
    for b in host_batches:
        dev_batches.append({k: to_t(v, False) for k, v in b.items()})
        hb = b
        if w["kind"] == "tpcc":  # host leg ships compact TPC-C records (LTPG_BATCH_COMPACT_PARAMS)
            packed, offs = ltpg.pack_params_compact(b["type"], b["params"])
            # consecutive TIDs ship as the first one (LTPG_BATCH_TID_RANGE); a shard's are not consecutive
            hb = {"tid": b["tid"] if sharded else b["tid"][:1].copy(), "type": b["type"], "params": packed,
                  "offsets": offs}
            if sharded:
                hb.update(grank=b["grank"], n_global=b["n_global"])
        pin_batches.append({k: to_t(v, True) for k, v in hb.items()})
        if w["kind"] == "tpcc":
            pin_batches[-1]["compact"] = True
            pin_batches[-1]["tid_range"] = not sharded

    # result buffers allocated once (device for the resident leg, pinned host for e2e), so no
    # allocation ever lands inside a timed step
    n_reads = B * w["ops"] if w["kind"] == "ycsb" else 4 * B
    dev_out = db._outputs(B, n_reads, True)
    def pinned_out():
        return {"status": torch.empty(B, dtype=torch.uint8).pin_memory(),
                "commit_bits": torch.empty((B + 31) // 32, dtype=torch.int32).pin_memory(),
                "abort_idx": torch.empty(B, dtype=torch.int32).pin_memory(),
                "n_aborted": torch.zeros(1, dtype=torch.int32).pin_memory(),
                "reads": torch.empty(n_reads, dtype=torch.int64).pin_memory()}
    pin_outs = [pinned_out() for _ in range(3)]  # three batches in flight in the e2e pipeline

    def run(bd, bh, clock, device, stats, wait=True, slot=0):
        inputs = bd if device else bp_of(bh)
        out = dev_out if device else pin_outs[slot]
        if w["kind"] == "ycsb":
            return db.run_ops(inputs, stream=torch.cuda.current_stream().cuda_stream, want_reads=True,
                              device_out=device, stats=stats, n_txns=len(bh["tid"]), n_ops=len(bh["args"]),
                              out=out, wait=wait)
        # host outputs: the commit bitmask, the abort list and the COMMITTED txns' result slots (written
        # into pinned host memory by the kernel, LTPG_RESULT_COMMITTED_READS; the slots of aborted
        # txns are snapshot reads recomputed on retry); status only for a shard (commit counting)
        return db.run_tpcc(inputs, clock, stream=torch.cuda.current_stream().cuda_stream, want_reads=True,
                           device_out=device, stats=stats, n_txns=len(bh["tid"]), out=out, wait=wait,
                           committed_reads=not device, no_status=not device and not sharded)

    pin_of = {id(h): p for h, p in zip(host_batches, pin_batches)}

    def bp_of(bh):
        return pin_of[id(bh)]

    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    clock = 2
    if not os.environ.get("LTPG_NO_CLOCKS"):
        clk.ready.wait(30)  # NVML init on a fresh box can take seconds
    for s in range(args.warmup):
        i = s % n_distinct
        run(dev_batches[i], host_batches[i], clock, True, False)
        clock += 1
    torch.cuda.synchronize()
    if dist:
        dist.barrier()

    # ---- timed: device-resident inputs ------------------------------------------------------
    # The timed batches run without per-stage instrumentation (ltpg_stats records 7 events per
    # batch: ~40 us on the small configs); commits are counted from the status array after each
    # step's end event.  A second, untimed pass over the same batches collects the stage split
    # (roofline kernel time) and the kernel count.
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    commits, procs, exec_ms, kernels, stage = [], [], [], 0, []
    torch.cuda.synchronize()
    tw0 = time.time()
    for s in range(args.steps):
        i = (args.warmup + s) % n_distinct
        flush.fill_(s & 0xFF)  # evict L2 between steps (outside the timed events)
        ev[s][0].record(stream)
        # submitted asynchronously and completed after the end event: the event pair brackets the
        # batch's device work (its last node is the result publish), not the host's wake-up from
        # the completion wait
        pend = run(dev_batches[i], host_batches[i], clock, True, False, wait=False)
        ev[s][1].record(stream)
        out = pend.wait()
        clock += 1
        n_s = len(host_batches[i]["tid"])
        if sharded:  # the commits of the txns this rank is home of (summed over ranks below)
            commits.append(int(((out["status"][:n_s] == 1) & home_dev[i]).sum()))
        else:
            commits.append(int((out["status"][:n_s] == 1).sum()))
        procs.append(n_s)
    torch.cuda.synchronize()
    clk.mark(tw0, time.time())
    step_ms = [a.elapsed_time(b) for a, b in ev]
    for s in range(args.steps):  # instrumented pass (not timed for the value)
        i = (args.warmup + s) % n_distinct
        flush.fill_(s & 0xFF)
        out = run(dev_batches[i], host_batches[i], clock, True, True)
        clock += 1
        st = out["stats"]
        exec_ms.append(st["ms_group"] if (fused_front or single) else st["ms_exec"])
        kernels += st["n_kernels"]
        stage.append(st)
    if os.environ.get("LTPG_BENCH_DEBUG"):
        log("step ms:", ["%.3f" % x for x in step_ms])
        log("lib ms :", ["%.3f" % sum(st_[k] for k in st_ if k.startswith("ms_")) for st_ in stage])
    total_s = sum(step_ms) / 1000.0
    # global batches: the verdicts are exchanged, every rank reports the same commits -- count
    # them once; sharded: every rank counts its home txns -- sum; time = max over ranks
    all_commits, all_procs = float(sum(commits)), float(sum(procs))
    if sharded:
        t = torch.tensor([all_commits], dtype=torch.float64, device="cpu" if shared else dev)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        all_commits = float(t.item())
        all_procs = float(B * args.steps)
    if dist:
        t = torch.tensor([total_s], device="cpu" if shared else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_s = float(t.item())
    value = all_commits / total_s

    # ---- timed: end to end through the public API, pinned host buffers ------------------------
    # Inter-batch pipeline (NEXT-2): batch s is submitted asynchronously while batch s-1
    # computes; the library uploads on one copy stream and downloads on another.  Every step's
    # H2D of its inputs and D2H of its results are inside the timed region (first submit to
    # last completion).  Inputs and state are larger than L2 for the large configs.
    # ---- closed loop with retries (a9): each step's batch = the previous step's
    # conflict aborts (original TIDs, ltpg_compose_retry) + fresh txns from a pool; composition
    # and upload happen between the timed batches (device time only, like the leg above) ----
    closed = None
    if world == 1 and not args.no_closed_loop:
        pool = host_batches[0]
        for hb in host_batches[1:]:  # one TID-ordered pool of fresh txns
            if w["kind"] == "ycsb":
                pool = {"tid": np.concatenate([pool["tid"], hb["tid"]]), "ops": np.concatenate([pool["ops"], hb["ops"]]),
                        "args": np.concatenate([pool["args"], hb["args"]]),
                        "op_begin": np.concatenate([pool["op_begin"], hb["op_begin"][1:] + pool["op_begin"][-1]]).astype(np.uint32)}
            else:
                pool = {k: np.concatenate([pool[k], hb[k]]) for k in ("tid", "type", "params")}
        def pool_from(c):
            if w["kind"] == "ycsb":
                ob = pool["op_begin"]
                return {"tid": pool["tid"][c:], "ops": pool["ops"][ob[c]:], "args": pool["args"][ob[c]:],
                        "op_begin": (ob[c:] - ob[c]).astype(np.uint32)}
            return {k: pool[k][c:] for k in ("tid", "type", "params")}
        max_ops = B * w["ops"] if w["kind"] == "ycsb" else 0
        cur, cursor = pool_from(0), 0
        cur, nf = ltpg.compose_retry(cur, np.zeros(0, np.uint32), cur, B, max_ops)  # first batch: fresh only
        cursor += nf
        c_ms, c_commit, c_retried, c_steps = 0.0, 0, 0, 0
        for s_ in range(args.steps):
            bd = {k: to_t(v, False) for k, v in cur.items()}
            flush.fill_(s_ & 0xFF)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            pend = run(bd, cur, clock, True, False, wait=False)
            e1.record(stream)
            outc = pend.wait()
            clock += 1
            torch.cuda.synchronize()
            c_ms += e0.elapsed_time(e1)
            st_h = outc["status"][:len(cur["tid"])].cpu().numpy()
            c_commit += int((st_h == 1).sum())
            c_steps += 1
            ab = np.nonzero(st_h == 0)[0].astype(np.uint32)
            if cursor >= len(pool["tid"]):
                break  # fresh pool used up
            nxt, nf = ltpg.compose_retry(cur, ab, pool_from(cursor), B, max_ops)
            c_retried += len(ab)
            cursor += nf
            cur = nxt
        closed = {"value": c_commit / (c_ms / 1000.0), "unit": UNIT, "steps": c_steps,
                  "ms_per_step": c_ms / c_steps, "commit_rate": c_commit / (c_steps * B),
                  "retried_per_step": c_retried / max(c_steps - 1, 1),
                  "note": "next batch = aborts (original TIDs) + fresh txns (ltpg_compose_retry); device time "
                          "per batch, composition and upload outside the timed region"}

    # ---- closed loop END TO END (batches back to back, aborts re-run in the next batch):
    # every step = the previous step's conflict aborts, carried on the device
    # (LTPG_BATCH_CARRY_ABORTS, a9 without a host round trip) + as many fresh txns as fit, taken
    # from a pool of pinned compact client records.  Timed per step (CUDA events on the stream +
    # wall clock): the host's submission (slice of the pool, its offsets rebased into a pinned
    # buffer), H2D of the fresh records, every kernel, D2H of status / bitmask / abort list / all
    # result slots.  TPC-C, single GPU. ----
    closed_e2e = None
    if world == 1 and w["kind"] == "tpcc" and not args.no_closed_loop and not args.no_e2e:
        pool = {k: np.concatenate([hb[k] for hb in host_batches]) for k in ("tid", "type", "params")}
        ppk, poffs = ltpg.pack_params_compact(pool["type"], pool["params"])
        pin = {"tid": to_t(pool["tid"], True), "type": to_t(pool["type"], True), "params": to_t(ppk, True)}
        offs_pin = torch.empty(B + 1, dtype=torch.int32).pin_memory()
        offs_np = offs_pin.numpy().view(np.uint32)
        out_c = pin_outs[0]
        torch.cuda.synchronize()
        cursor, c_commit, c_carried, c_steps, h2d_c, d2h_c = 0, 0, 0, 0, 0, 0
        ce0, ce1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        tw0 = time.time()
        ce0.record(stream)
        for s_ in range(args.steps):
            nc = db.pending_aborts() if s_ else 0
            m = min(B - nc, len(pool["tid"]) - cursor)
            if m <= 0:
                break
            np.subtract(poffs[cursor:cursor + m + 1], poffs[cursor], out=offs_np[:m + 1])
            p0, p1 = int(poffs[cursor]), int(poffs[cursor + m])
            inp = {"tid": pin["tid"][8 * cursor:8 * (cursor + m)], "type": pin["type"][cursor:cursor + m],
                   "params": pin["params"][p0:p1], "offsets": offs_pin[:m + 1], "compact": True}
            outc = db.run_tpcc(inp, clock, stream=stream.cuda_stream, want_reads=True, device_out=False,
                               n_txns=m, out=out_c, carry=s_ > 0, committed_reads=True, no_status=True,
                               no_abort_list=True)
            clock += 1
            n_s = nc + m
            nc_s = int(np.bitwise_count(np.asarray(outc["commit_bits"])[:(n_s + 31) // 32].view(np.uint32)).sum())
            c_commit += nc_s
            c_carried += nc
            c_steps += 1
            h2d_c += 8 * m + m + (p1 - p0) + 4 * (m + 1)
            d2h_c += 4 * ((n_s + 31) // 32) + 32 * nc_s + 68  # bitmask, committed txns' slots, counters
            cursor += m
        ce1.record(stream)
        torch.cuda.synchronize()
        wall = time.time() - tw0
        clk.mark(tw0, time.time())
        c_s = ce0.elapsed_time(ce1) / 1000.0
        closed_e2e = {"value": c_commit / c_s, "unit": UNIT, "steps": c_steps, "ms_per_step": 1000 * c_s / c_steps,
                      "wall_ms_per_step": 1000 * wall / c_steps, "commit_rate": c_commit / (c_steps * B),
                      "carried_per_step": c_carried / max(c_steps - 1, 1),
                      "h2d_bytes_per_step": h2d_c // c_steps, "d2h_bytes_per_step": d2h_c // c_steps,
                      "note": "closed loop end to end: previous step's aborts carried on the device "
                              "(LTPG_BATCH_CARRY_ABORTS) + fresh compact records from pinned host memory; "
                              "returns the commit bitmask and the committed txns' result slots "
                              "(LTPG_RESULT_COMMITTED_READS, written into pinned host memory by the kernel); "
                              "H2D, kernels, D2H and host submission inside the timed region"}

    e2e = None
    if not args.no_e2e:
        e_commits = []
        h2d = d2h = 0
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        tw0 = time.time()
        e0.record(stream)
        inflight = []

        def collect(p):
            nonlocal d2h
            out = p.wait()
            n = shard_sizes[p.i]  # (the pinned output buffers are sized for the full batch)
            # commits: popcount of the returned commit bitmask (no per-stage instrumentation)
            cb = out["commit_bits"]
            cb = cb.numpy() if hasattr(cb, "numpy") else cb
            if sharded:  # the commits of this rank's home txns (status is downloaded anyway)
                st_ = out["status"]
                st_ = st_.numpy() if hasattr(st_, "numpy") else st_
                e_commits.append(int(((st_[:n] == 1) & home_masks[p.i]).sum()))
            else:
                e_commits.append(int(np.bitwise_count(cb[:(n + 31) // 32].view(np.uint32)).sum()))
            nreads = n_reads if w["kind"] == "ycsb" else 4 * n
            if w["kind"] == "tpcc":  # bitmask, abort list (copied at capacity), committed slots, counters
                d2h += 4 * ((n + 31) // 32) + 4 * n + 32 * e_commits[-1] + 68 + (n if sharded else 0)
            else:
                d2h += n + 4 * ((n + 31) // 32) + 4 * n + 8 * nreads + 68

        for s in range(args.steps):
            i = (args.warmup + s) % n_distinct
            bh = host_batches[i]
            inflight.append(run(None, bh, clock, False, False, wait=False, slot=s % 3))
            inflight[-1].i = i
            clock += 1
            h2d += sum(v.nbytes for v in bp_of(bh).values() if hasattr(v, "nbytes"))
            if len(inflight) == 3:  # keep two batches queued behind the one completing
                collect(inflight.pop(0))
        while inflight:
            collect(inflight.pop(0))
        e1.record(stream)
        torch.cuda.synchronize()
        clk.mark(tw0, time.time())
        e_s = e0.elapsed_time(e1) / 1000.0
        e_c = float(sum(e_commits))
        if sharded:
            t = torch.tensor([e_c], dtype=torch.float64, device="cpu" if shared else dev)
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
            e_c = float(t.item())
        if dist:
            t = torch.tensor([e_s], device="cpu" if shared else dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_s = float(t.item())
        e2e = {"value": e_c / e_s, "unit": UNIT, "h2d_bytes_per_step": h2d // args.steps,
               "d2h_bytes_per_step": d2h // args.steps, "ms_per_step": 1000 * e_s / args.steps,
               "pipeline": "3 batches in flight (LTPG_BATCH_ASYNC): H2D / kernels / D2H overlapped",
               "input": ("compact TPC-C records (LTPG_BATCH_COMPACT_PARAMS) expanded on the GPU, consecutive "
                         "TIDs as their first one (LTPG_BATCH_TID_RANGE)"
                         if w["kind"] == "tpcc" else "16-byte op records + i64 args"),
               "output": ("commit bitmask + abort list + the committed txns' result slots "
                          "(LTPG_RESULT_COMMITTED_READS | LTPG_RESULT_NO_STATUS)" if w["kind"] == "tpcc"
                          else "status + bitmask + abort list + every op's result slot")}

    if not os.environ.get("LTPG_NO_CLOCKS"):
        clk.__exit__(None, None, None)
    if rank != 0:
        if dist:
            dist.barrier()
            dist.destroy_process_group()
        return

    # ---- roofline of the dominant kernel (execute) ------------------------------------------------
    peak, peak_kind = measured_peaks()
    roof = None
    if w["kind"] == "ycsb":
        model = fused_algorithmic_bytes if fused_front else exec_algorithmic_bytes
        kname = "k_ops_small" if single else "k_ops_fused" if fused_front else "k_ops_exec"
        bytes_exec = statistics.mean(model(host_batches[(args.warmup + s) % n_distinct], w.get("sparse", False))
                                     for s in range(args.steps))
        ms = statistics.mean(exec_ms)
        ach = bytes_exec / (ms / 1000.0) / 1e9
        roof = {"bound": "hbm", "kernel": kname, "achieved": ach, "peak": peak, "unit": "GB/s",
                "frac": ach / peak, "traffic": ncu_traffic(name, kname), "peak_source": peak_kind,
                "algorithmic_bytes_per_launch": bytes_exec, "kernel_ms": ms,
                "kernel_share_of_step": ms / statistics.mean(step_ms)}
        nrand = statistics.mean(ops_random_reads(host_batches[(args.warmup + s) % n_distinct], w.get("sparse", False))
                                for s in range(args.steps))
        roof["random_access"] = {
            "reads_per_launch": nrand, "ceiling_g_per_s": RANDOM_READ_CEILING_G,
            "achieved_g_per_s": nrand / (ms / 1000.0) / 1e9,
            "frac": nrand / (ms / 1000.0) / 1e9 / RANDOM_READ_CEILING_G,
            "source": "tools/randbw.cu, profiles/randbw_r01.txt"}
    else:
        bytes_exec = statistics.mean(tpcc_exec_algorithmic_bytes(host_batches[(args.warmup + s) % n_distinct],
                                                                  w["mode"]) for s in range(args.steps))
        ms = statistics.mean(exec_ms)
        ach = bytes_exec / (ms / 1000.0) / 1e9
        kname = "k_tpcc_small" if single else "k_tpcc_phase<PH_EXEC>"
        roof = {"bound": "hbm", "kernel": kname, "achieved": ach, "peak": peak, "unit": "GB/s",
                "frac": ach / peak, "traffic": ncu_traffic(name, "k_tpcc_small" if single else "k_tpcc_phase<0,"),
                "peak_source": peak_kind,
                "algorithmic_bytes_per_launch": bytes_exec, "kernel_ms": ms,
                "kernel_share_of_step": ms / statistics.mean(step_ms)}
        ntouch = statistics.mean(tpcc_random_touches(host_batches[(args.warmup + s) % n_distinct])
                                 for s in range(args.steps))
        roof["random_access"] = {
            "touches_per_launch": ntouch, "ceiling_g_per_s": RANDOM_READ_CEILING_G,
            "achieved_g_per_s": ntouch / (ms / 1000.0) / 1e9,
            "frac": ntouch / (ms / 1000.0) / 1e9 / RANDOM_READ_CEILING_G,
            "source": "tools/randbw.cu, profiles/randbw_r01.txt; touches: bench.py tpcc_random_touches"}
    if single:  # the one launch also detects, writes back and finalises: its execute-stage bytes
        roof["note"] = ("single cooperative launch (the whole batch): achieved counts only the execute-stage "
                        "algorithmic bytes over the whole kernel time -- a lower bound; the kernel is bound by "
                        "dependent cold-L2 round trips per stage, not by HBM bandwidth (DESIGN.md 6b)")

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1000 * total_s / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "config": dict(config_of(name), parallelism=(
                ("%d ranks by warehouse range, SHARDED global batch (each rank gets the txns touching its "
                 "warehouses; verdict bytes of cross-rank txns over peer memory, csrc/xchg.cu)" % world)
                if sharded else
                ("%d ranks by key range, same global batch on every rank, per-txn verdict planes over peer "
                 "memory (csrc/xchg.cu)" % world) if world > 1 else "single GPU")),
            "clocks": clk.summary(), "e2e": e2e, "closed_loop": closed, "closed_loop_e2e": closed_e2e, "gpu_launches": kernels, "roofline": roof,
            "commit_rate": all_commits / all_procs, "processed_txns_per_s": all_procs / total_s,
            "stage_ms_mean": {k: statistics.mean(s_[k] for s_ in stage)
                              for k in ("ms_upload", "ms_group", "ms_exec", "ms_detect", "ms_writeback",
                                        "ms_download")}}
    if args.flags:
        line["config"]["flags"] = args.flags
    line["gpus_requested"] = args.gpus
    line["gpus_active"] = min(world, ndev)
    line["ranks"] = world
    line["exchange"] = (None if world == 1 else "peer-memory stores + signals (csrc/xchg.cu)" +
                        (", sharded batches" if sharded else ", global batches"))
    if sharded:
        line["shard_txns_rank0"] = statistics.mean(shard_sizes)
    if shared:
        line["config"]["devices"] = ("%d ranks on %d GPU(s): functional check of the multi-rank path, "
                                     "not a scaling number" % (world, ndev))
    if world == 1 and not args.no_cpu_baseline:
        try:
            line["cpu_baseline"] = cpu_baseline(name)
        except Exception as e:  # never lose the GPU number to the baseline leg
            line["cpu_baseline"] = {"error": repr(e)}
    print(json.dumps(line), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
