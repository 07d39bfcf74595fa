#!/usr/bin/env python
"""Benchmark of the merge-path hot path on B200 (BASELINE.json metric).

Headline (the driver's JSON line): a step = one pass of the whole hot path
over the C2 workload (BJ:8, configs[1], the config BASELINE.json's metric is
quoted on): SpMV y = A x, SpAdd C = A + A^T (the one-pass msp_spadd_fused)
and SpGEMM C = A A (setup + symbolic + numeric) on the 3-D 27-point Poisson
matrix 100^3 in fp64.
`value` is the SpMV achieved GB/s (algorithmic bytes / time).

Beside it, in the same line:
  * `table`: every BASELINE.json config at full size with its BJ ops --
    SpMV (ms, GB/s, fraction of measured HBM, GFLOP/s), SpAdd A + A^T
    (C1, C3 fp32: input nnz/s, GB/s, fraction; two-phase symbolic + numeric
    and the one-pass form) and SpGEMM A * A (C1, C2,
    C4, C5: products/s and per-pass ms and algorithmic GB/s for setup /
    symbolic / numeric);
  * `predictability`: R^2 and Pearson rho of time ~ work over the configs
    (SpMV vs nnz over C1-C5 and over C1-C4, SpGEMM vs Nprods);
  * `cpu_baseline`: the CPU oracle (test infrastructure, as it stands) on the
    host: SpMV C2 single-threaded (the reported value), and SpMV C2, SpAdd C3
    and SpGEMM C2 on bounded row samples with 1 process and with one
    process per host core (row blocks of the same calls), with nproc and the
    CPU model.

Multi-GPU (torchrun, N > 1): the headline is weak scaling -- rank r owns a
100^3 slab of a 100 x 100 x (100 N) Poisson grid (nnz-balanced row blocks), x
is all-gathered over NCCL before the local SpMV and B = A's row blocks are
all-gathered before the local SpGEMM; `c5_strong` adds BJ's
multi-GPU config C5 row-partitioned across the N ranks (strong scaling) with
the all-gather times reported separately.  Timing is the max over ranks.

--impl reference times the CPU oracle (the plain C reference written from the
paper) on the host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import subprocess
import sys
import threading
import time
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent
sys.path.insert(0, str(ROOT))

HBM_FALLBACK = 6650.0
METRIC = "SpMV GB/s (algorithmic bytes / time) on C2; SpAdd input nnz/s, SpGEMM products/s beside"
WORKLOAD_C2 = "C2: 3D Poisson 27-point 100^3 fp64 (BJ:8)"
BJ_OPS = {"C1": ("spmv", "spadd", "spgemm"), "C2": ("spmv", "spgemm"), "C3": ("spmv", "spadd"),
          "C4": ("spmv", "spgemm"), "C5": ("spmv", "spgemm")}
L2_BYTES = 126 * 2 ** 20


def peaks():
    try:
        d = json.loads((ROOT / "MEASURED_PEAKS.json").read_text())
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return HBM_FALLBACK, "fallback"


# --------------------------------------------------------------- clocks

class ClockSampler:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md)."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.th = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return

        def rd():
            for ln in self.proc.stdout:
                self.rows.append([c.strip() for c in ln.split(",")])
        self.th = threading.Thread(target=rd, daemon=True)
        self.th.start()

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        if self.th:
            self.th.join(timeout=1)
        sm = [float(r[0]) for r in self.rows if r and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for k, nm in enumerate(names):
                if len(r) > 3 + k and r[3 + k].lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------- algorithmic bytes

def spmv_alg_bytes(m, n, nnz, vsize):
    """4 (col) + s (val) per nonzero, 4 (offset) + s (y) per row, s (x) per
    column read once; plus the final row offset."""
    return nnz * (4 + vsize) + m * (4 + vsize) + 4 + n * vsize


def spadd_alg_bytes(m, nnz_a, nnz_b, nnz_c, vsize):
    """Input nonzeros read (4 + s), output nonzeros written (4 + s), three
    row-offset arrays per row (A, B read; C written)."""
    return (nnz_a + nnz_b) * (4 + vsize) + nnz_c * (4 + vsize) + 3 * 4 * (m + 1)


def spgemm_pass_bytes(m, nnz_a, nprods, nnz_c, vsize, rowacc=False, small=False):
    """The method's own traffic per pass.  Small-row path
    (small, every short row has few products): setup as below plus the B row
    start of every A nonzero (4) and the row classification (A offsets and 16
    of S per row).  Symbolic = expand (per A nonzero: COO row, B row start,
    S[j], S[j+1], row mode: 4 + 4 + 16 + 1; per product: one B column
    gathered (4) and staged (4)) + compress (per product: the staged column
    (4); per row: mode, A offsets, S, the count written: 1 + 8 + 16 + 4).
    Numeric = expand (the same per A nonzero plus a_ij (s); per product a B
    value gathered (s) and the fp64 product staged (8)) + compress (per
    product: staged product (8) and column (4) read; per row: mode, A
    offsets, S, C offsets; C written (4 + s per C nonzero)).
    Row accumulator (rowacc): setup as below plus the span pass (A columns,
    8 of B offsets and 8 of B columns per A nonzero); symbolic reads A columns and B offsets
    (12 per A nonzero), gathers one B column per product (4) and writes each
    row's column list (4 per C nonzero); numeric reads the same plus A values
    (12 + s per A nonzero), gathers a B column + value per product (4 + s),
    reads the column list (4 per C nonzero) and writes C (4 + s).
    ESC:
    setup    -- A offsets + columns read, B offsets gathered (8 per A
                nonzero), S written (8), COO rows written (4);
    symbolic -- A columns, COO rows and S read (16 per A nonzero), one B
                column gathered per product (4), the 2-byte tile permutation
                written per product, C row offsets written;
    numeric  -- A columns + values, rows and S read (16 + s per A nonzero),
                one B column + value gathered per product (4 + s), the
                permutation read (2), C columns + values written (4 + s)."""
    setup = 4 * (m + 1) + nnz_a * (4 + 8 + 8 + 4)
    if small:
        # expand + compress: the expand pass writes each product's column
        # (symbolic, 4) or fp64 product (numeric, 8) to a staging array that
        # the compress pass reads back (numeric also reads the columns)
        setup += nnz_a * 4 + m * (8 + 16)
        symbolic = nnz_a * (4 + 4 + 16 + 1) + nprods * (4 + 4 + 4) + m * (1 + 8 + 16 + 4)
        numeric = (nnz_a * (4 + 4 + 16 + 1 + vsize) + nprods * (vsize + 8 + 8 + 4) + nnz_c * (4 + vsize)
                   + m * (1 + 8 + 16 + 8))
        return {"setup": setup, "symbolic": symbolic, "numeric": numeric}
    if rowacc:
        setup += 4 * (m + 1) + nnz_a * (4 + 8 + 8)
        symbolic = nnz_a * 12 + nprods * 4 + nnz_c * 4 + 4 * (m + 1)
        numeric = nnz_a * (12 + vsize) + nprods * (4 + vsize) + nnz_c * (4 + 4 + vsize) + 4 * (m + 1)
        return {"setup": setup, "symbolic": symbolic, "numeric": numeric}
    symbolic = nnz_a * 16 + nprods * (4 + 2) + 4 * (m + 1)
    numeric = nnz_a * (16 + vsize) + nprods * (4 + vsize + 2) + nnz_c * (4 + vsize) + 4 * (m + 1)
    return {"setup": setup, "symbolic": symbolic, "numeric": numeric}


_GEN = {}


def config_matrix(name, mode="random"):
    """gen.config, memoised (the table and the CPU baseline share inputs)."""
    import gen
    key = (name, mode)
    if key not in _GEN:
        _GEN[key] = gen.config(name, mode)
    return _GEN[key]


def transposed(name):
    import gen
    key = (name, "T")
    if key not in _GEN:
        _GEN[key] = gen.transpose(config_matrix(name))
    return _GEN[key]


def fit(xs, ys):
    """Least-squares time ~ work: R^2 and Pearson rho."""
    x = np.asarray(xs, float)
    y = np.asarray(ys, float)
    if x.size < 3:
        return None
    A = np.vstack([x, np.ones_like(x)]).T
    coef, *_ = np.linalg.lstsq(A, y, rcond=None)
    pred = A @ coef
    ss_res = float(np.sum((y - pred) ** 2))
    ss_tot = float(np.sum((y - y.mean()) ** 2))
    return {"r2": 1 - ss_res / ss_tot if ss_tot > 0 else 1.0, "rho": float(np.corrcoef(x, y)[0, 1]),
            "slope_ms_per_unit": float(coef[0]), "intercept_ms": float(coef[1]), "n": int(x.size)}


# --------------------------------------------------------------- CLI

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="msp", choices=["msp", "reference"])
    ap.add_argument("--ops", default="spmv,spadd,spgemm")
    ap.add_argument("--spmv-reps", type=int, default=20, help="SpMV launches per step (timed individually)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-table", action="store_true", help="skip the per-config table (C1..C5)")
    ap.add_argument("--table-configs", default="C1,C2,C3,C4,C5")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return reference_arm(args)
    return msp_arm(args)


# --------------------------------------------------------------- CPU oracle (test infrastructure)

def _cpu_info():
    model = platform.processor() or ""
    try:
        for ln in Path("/proc/cpuinfo").read_text().splitlines():
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return os.cpu_count() or 1, model


_POOL_STATE = {}


def _pool_call(job):
    """Worker body (fork): one row block of one oracle call."""
    import oracle
    kind, rows = job
    st = _POOL_STATE
    t0 = time.perf_counter()
    if kind == "spmv":
        oracle.spmv(st["A"], st["x"], rows)
    elif kind == "spadd":
        oracle.spadd_rows(st["A3"], st["T3"], rows)
    else:
        oracle.spgemm_rows(st["A"], st["A"], rows)
    return time.perf_counter() - t0


def _timed_parallel(kind, rows, procs):
    """Wall time of the oracle over `rows` split in `procs` contiguous blocks,
    one forked process per block (the oracle itself is unchanged)."""
    import multiprocessing as mp
    blocks = [b for b in np.array_split(rows, procs) if b.size]
    if procs == 1:
        t0 = time.perf_counter()
        _pool_call((kind, rows))
        return time.perf_counter() - t0
    ctx = mp.get_context("fork")
    with ctx.Pool(procs) as pool:
        pool.map(_pool_call, [(kind, blocks[0][:1])] * procs)  # warm the workers
        t0 = time.perf_counter()
        pool.map(_pool_call, [(kind, b) for b in blocks])
        return time.perf_counter() - t0


def cpu_baseline(budget_s=10.0, extended=True):
    """The oracle as it stands on this host: SpMV C2 single-threaded (value),
    plus bounded samples of SpMV C2, SpAdd C3 and SpGEMM C2 at 1 process and
    at one process per core."""
    import gen
    import oracle
    nproc, model = _cpu_info()
    A = config_matrix("C2")
    x = gen.x_vector(A.n, "random", seed=1002)
    oracle.spmv(A, x)  # warm
    t0 = time.perf_counter()
    reps = 0
    while time.perf_counter() - t0 < budget_s:
        oracle.spmv(A, x)
        reps += 1
    dt = (time.perf_counter() - t0) / reps
    by = spmv_alg_bytes(A.m, A.n, A.nnz, 8)
    res = {"value": by / dt / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
           "sample": f"full C2 SpMV x{reps} in {reps * dt:.1f}s (single-threaded C oracle)",
           "ms_per_spmv": dt * 1e3, "nproc": nproc, "cpu_model": model}
    if not extended:
        return res
    ops = {}
    _POOL_STATE.update(A=A, x=x)
    rows_all = np.arange(A.m, dtype=np.int32)
    for procs in sorted({1, nproc}):
        s = _timed_parallel("spmv", rows_all, procs)
        ops.setdefault("spmv_C2", {})[f"p{procs}"] = {"s": s, "GB_s": by / s / 1e9,
                                                       "sample": "all 10^6 rows of C2"}
    # SpGEMM C2: a contiguous 1/40 of the rows (about 17.6M products)
    rows = np.arange(0, A.m // 40, dtype=np.int32)
    npr = int(oracle.nprods(gen.CSR(rows.size, A.n, A.rp[:rows.size + 1], A.col[:A.rp[rows.size]],
                                    A.val[:A.rp[rows.size]]), A))
    for procs in sorted({1, nproc}):
        s = _timed_parallel("spgemm", rows, procs)
        ops.setdefault("spgemm_C2", {})[f"p{procs}"] = {"s": s, "products_per_s": npr / s,
                                                         "sample": f"rows [0, {rows.size}) of C2 A*A, {npr} products"}
    # SpAdd C3 fp32 A + A^T: a contiguous 1/16 of the rows
    A3 = config_matrix("C3")
    T3 = transposed("C3")
    _POOL_STATE.update(A3=A3, T3=T3)
    r3 = np.arange(0, A3.m // 16, dtype=np.int32)
    nin = int(A3.rp[r3.size] + T3.rp[r3.size])
    for procs in sorted({1, nproc}):
        s = _timed_parallel("spadd", r3, procs)
        ops.setdefault("spadd_C3", {})[f"p{procs}"] = {"s": s, "input_nnz_per_s": nin / s,
                                                        "sample": f"rows [0, {r3.size}) of C3 A+A^T, {nin} input nnz"}
    res["ops"] = ops
    res["all_cores"] = {"procs": nproc, "spmv_GB_s": ops["spmv_C2"][f"p{nproc}"]["GB_s"]}
    return res


def reference_arm(args):
    """The reference arm: the CPU oracle as it stands, on the host cores, on
    the msp arm's config / metric / unit (bounded samples)."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    res = cpu_baseline(budget_s=max(2.0, 6.0 * (args.steps + args.warmup) / 20), extended=False)
    line = {"impl": "reference", "metric": METRIC, "value": res["value"],
            "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded generators, gen/)",
            "config": {"workload": WORKLOAD_C2, "kernel": "CPU oracle (scalar CSR, P:364-370), host cores"},
            "cpu_baseline": res, "e2e": {"value": res["value"], "unit": "GB/s", "h2d_bytes_per_step": 0,
                                          "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


# --------------------------------------------------------------- msp arm

def workload(rank: int, world: int):
    """C2 (world == 1) or this rank's 100^3 slab of a 100x100x(100*world) grid."""
    import gen
    if world == 1:
        A = config_matrix("C2")
        return A, 0, A.m
    G = gen.poisson3d_27pt(100, 100, 100 * world)
    G = G.with_values(gen.matrices.random_values(G.nnz, 1002))
    from paper_conf_ipps_daltonbmog15_b200 import row_split  # libmsp host helper
    starts = row_split(G.rp, world)
    return G, int(starts[rank]), int(starts[rank + 1])


def ncu_traffic(world):
    """DRAM bytes per launch of the SpMV kernel on C2 from the committed ncu
    --set full capture (dram__bytes_read.sum + dram__bytes_write.sum)."""
    try:
        d = json.loads((ROOT / "profiles" / "spmv_C2_ncu_full.json").read_text())
        if world != 1:
            return {"traffic": None, "traffic_source": "ncu capture is of the 1-GPU C2 launch"}
        return {"traffic": float(d["dram_bytes_per_launch"]),
                "traffic_source": f"profiles/spmv_C2_ncu_full.json ({d.get('source', 'ncu --set full')})"}
    except Exception as e:  # noqa: BLE001
        return {"traffic": None, "traffic_source": f"unavailable: {e}"}


def spmv_kernel_name(m, nnz):
    """The SpMV kernel libmsp picks for this matrix: warp tiles
    with row-aligned lanes when the mean row length is >= 20, else the
    CTA-tile transpose walk."""
    return "spmv_wt_kernel" if m > 0 and nnz >= 20 * m else "spmv_merge_kernel"


class Timer:
    """CUDA events on the launching stream."""

    def __init__(self, torch, stream):
        self.torch, self.stream = torch, stream

    def ev(self):
        e = self.torch.cuda.Event(enable_timing=True)
        e.record(self.stream)
        return e


def table_configs(msp, torch, dev, names, peak, flush):
    """Every BASELINE.json config at full size with its BJ ops."""
    import gen
    stream = torch.cuda.current_stream(dev)
    tm = Timer(torch, stream)
    out = {}
    for name in names:
        t_gen = time.time()
        A = config_matrix(name)
        gen_s = time.time() - t_gen
        vs = A.val.dtype.itemsize
        dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), dev)
        ent = {"m": A.m, "nnz": A.nnz, "dtype": str(A.val.dtype), "gen_s": round(gen_s, 1)}
        small = spmv_alg_bytes(A.m, A.n, A.nnz, vs) < 2 * L2_BYTES
        if "spmv" in BJ_OPS[name]:
            x = torch.as_tensor(gen.x_vector(A.n, "random", seed=1000 + int(name[1]), dtype=A.val.dtype), device=dev)
            y = torch.empty(A.m, dtype=x.dtype, device=dev)
            reps = 5 if name == "C5" else 20
            for _ in range(3):
                msp.spmv(dA, x, out=y)
            ts = []
            for _ in range(reps):
                if small:
                    flush()
                a = tm.ev()
                msp.spmv(dA, x, out=y)
                b = tm.ev()
                ts.append((a, b))
            torch.cuda.synchronize(dev)
            ms = float(np.mean([a.elapsed_time(b) for a, b in ts]))
            by = spmv_alg_bytes(A.m, A.n, A.nnz, vs)
            ent["spmv"] = {"ms": ms, "alg_bytes": by, "GB_s": by / ms / 1e6, "frac_hbm": by / ms / 1e6 / peak,
                           "GFLOP_s": 2 * A.nnz / ms / 1e6, "l2": "flushed" if small else "inputs > L2",
                           "kernel": spmv_kernel_name(A.m, A.nnz)}
            # f4(i) ablation: the paper's nnz-only split with row compaction
            for _ in range(2):
                msp.spmv_nnz_split(dA, x, out=y)
            ts = []
            for _ in range(reps):
                if small:
                    flush()
                a = tm.ev()
                msp.spmv_nnz_split(dA, x, out=y)
                b = tm.ev()
                ts.append((a, b))
            torch.cuda.synchronize(dev)
            ms2 = float(np.mean([a.elapsed_time(b) for a, b in ts]))
            ent["spmv_nnz_split"] = {"ms": ms2, "GB_s": by / ms2 / 1e6, "frac_hbm": by / ms2 / 1e6 / peak,
                                     "vs_merge_grid": ms / ms2}
            del x, y
        if "spadd" in BJ_OPS[name]:
            T = transposed(name)
            dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), dev)
            C = msp.spadd(dA, dT)
            reps = 10
            ts = []
            # C's arrays preallocated (as a serving caller would): the timed
            # region holds the library calls, not the allocator
            oc = torch.empty(C.nnz, dtype=torch.int32, device=dev)
            ov = torch.empty(C.nnz, dtype=dA.dtype, device=dev)
            p = msp.SpAddPlan(dA, dT)  # plan (host objects) outside the timed region
            p.symbolic()  # untimed warm-up of this plan's path
            p.numeric(col=oc, val=ov)
            torch.cuda.synchronize(dev)
            for _ in range(reps):
                if small:
                    flush()
                a = tm.ev()
                p.symbolic()
                b = tm.ev()
                p.numeric(col=oc, val=ov)
                c = tm.ev()
                ts.append((a, b, c))
            torch.cuda.synchronize(dev)
            sym = float(np.mean([a.elapsed_time(b) for a, b, _ in ts]))
            num = float(np.mean([b.elapsed_time(c) for _, b, c in ts]))
            ms = sym + num
            by = spadd_alg_bytes(A.m, A.nnz, T.nnz, C.nnz, vs)
            ent["spadd"] = {"op": "A + A^T", "ms": ms, "symbolic_ms": sym, "numeric_ms": num,
                            "input_nnz": A.nnz + T.nnz, "nnz_c": C.nnz,
                            "input_nnz_per_s": (A.nnz + T.nnz) / ms * 1e3, "alg_bytes": by,
                            "GB_s": by / ms / 1e6, "frac_hbm": by / ms / 1e6 / peak}
            # one-pass form (msp_spadd_fused): same result, C allocated at nnz(A) + nnz(B)
            cap = A.nnz + T.nnz
            fc = torch.empty(cap, dtype=torch.int32, device=dev)
            fv = torch.empty(cap, dtype=dA.dtype, device=dev)
            for _ in range(2):  # untimed: first launches of this value type's kernels load their modules
                msp.spadd_fused(dA, dT, col=fc, val=fv)
            torch.cuda.synchronize(dev)
            ts = []
            for _ in range(reps):
                if small:
                    flush()
                a = tm.ev()
                msp.spadd_fused(dA, dT, col=fc, val=fv)
                b = tm.ev()
                ts.append((a, b))
            torch.cuda.synchronize(dev)
            fms = float(np.mean([a.elapsed_time(b) for a, b in ts]))
            ent["spadd_fused"] = {"op": "A + A^T, one pass", "ms": fms,
                                  "input_nnz_per_s": (A.nnz + T.nnz) / fms * 1e3, "alg_bytes": by,
                                  "GB_s": by / fms / 1e6, "frac_hbm": by / fms / 1e6 / peak,
                                  "vs_two_phase": ms / fms}
            del dT, C, T, fc, fv, oc, ov
        if "spgemm" in BJ_OPS[name]:
            reps = 3 if name == "C5" else 5
            rec = []
            oc = ov = None  # C's arrays, preallocated after the first (untimed) call
            path = None
            for i in range(reps + 2):
                if small:
                    flush()
                a = tm.ev()
                p = msp.SpGemmPlan(dA, dA)
                p.setup()
                b = tm.ev()
                p.symbolic()
                c = tm.ev()
                Cg = p.numeric(col=oc, val=ov)
                d = tm.ev()
                if i >= 2:
                    rec.append((a, b, c, d))
                nprods, nnzc = p.nprods, Cg.nnz
                inf = p.info
                path = ("esc_tiles" if inf.row_accumulator == 0 else
                        "small_rows" if inf.bitmap_rows == 0 else
                        "row_accumulator" if inf.small_rows == 0 else "small_rows+row_accumulator")
                rows_by_path = {"small": int(inf.small_rows), "bitmap": int(inf.bitmap_rows),
                                "long": int(inf.long_rows), "segmented": int(inf.segmented_rows)}
                if oc is None:
                    oc, ov = Cg.col, Cg.val
                del Cg, p
            del oc, ov
            torch.cuda.synchronize(dev)
            ph = {k: float(np.mean([r[j].elapsed_time(r[j + 1]) for r in rec]))
                  for j, k in enumerate(("setup", "symbolic", "numeric"))}
            ms = sum(ph.values())
            pb = spgemm_pass_bytes(A.m, A.nnz, nprods, nnzc, vs, path == "row_accumulator", path == "small_rows")
            ent["spgemm"] = {"op": "A * A", "ms": ms, "nprods": nprods, "nnz_c": nnzc, "short_row_path": path,
                             "rows_by_path": rows_by_path,
                             "products_per_s": nprods / ms * 1e3,
                             "passes": {k: {"ms": ph[k], "alg_bytes": pb[k], "GB_s": pb[k] / ph[k] / 1e6,
                                            "frac_hbm": pb[k] / ph[k] / 1e6 / peak} for k in ph}}
        del dA
        if name in ("C4", "C5"):  # not needed by the CPU baseline
            _GEN.pop((name, "random"), None)
        torch.cuda.empty_cache()
        out[name] = ent
    return out


def predictability(table):
    res = {}
    pts = [(v["nnz"], v["spmv"]["ms"]) for v in table.values() if "spmv" in v]
    res["spmv_time_vs_nnz"] = fit(*zip(*pts)) if len(pts) >= 3 else None
    pts4 = [(v["nnz"], v["spmv"]["ms"]) for k, v in table.items() if "spmv" in v and k != "C5"]
    res["spmv_time_vs_nnz_without_C5"] = fit(*zip(*pts4)) if len(pts4) >= 3 else None
    pg = [(v["spgemm"]["nprods"], v["spgemm"]["ms"]) for v in table.values() if "spgemm" in v]
    res["spgemm_time_vs_nprods"] = fit(*zip(*pg)) if len(pg) >= 3 else None
    return res


def c5_strong(msp, torch, dist, dev, rank, world):
    """BJ:11 -- C5 row-partitioned across the ranks (strong scaling): x
    all-gather + local SpMV, B all-gather + local SpGEMM; max over ranks."""
    import gen
    from paper_conf_ipps_daltonbmog15_b200 import dist as mdist
    G = gen.config("C5", "random")
    starts = mdist.split_rows(G.rp, world)
    r0, r1 = int(starts[rank]), int(starts[rank + 1])
    blk = mdist.row_block(G.rp, G.col, G.val, r0, r1, G.n, dev)
    xs = mdist.x_slice_of(torch.as_tensor(gen.x_vector(G.n, "random", seed=1005), device=dev), rank, world)
    stream = torch.cuda.current_stream(dev)
    tm = Timer(torch, stream)
    rec = {"allgather_x": [], "spmv": [], "gather_B": [], "spgemm": []}
    for i in range(4):
        dist.barrier()
        a = tm.ev()
        xf = mdist.allgather_x(xs, G.n)
        b = tm.ev()
        msp.spmv(blk, xf)
        c = tm.ev()
        Bf = mdist.gather_csr_blocks(blk)
        d = tm.ev()
        p = msp.SpGemmPlan(blk, Bf)
        p.setup()
        p.symbolic()
        p.numeric()
        e = tm.ev()
        torch.cuda.synchronize(dev)
        if i >= 1:
            for k, (u, v) in zip(rec, ((a, b), (b, c), (c, d), (d, e))):
                rec[k].append(u.elapsed_time(v))
        del Bf, p, xf
    out = {}
    for k, v in rec.items():
        t = torch.tensor([float(np.mean(v))], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        out[f"{k}_ms"] = float(t.item())
    by = spmv_alg_bytes(G.m, G.n, G.nnz, 8)
    out["spmv_GB_s"] = by / ((out["allgather_x_ms"] + out["spmv_ms"]) * 1e-3) / 1e9
    out["spmv_compute_GB_s"] = by / (out["spmv_ms"] * 1e-3) / 1e9
    out["workload"] = f"C5 (BJ:11) {G.m} rows, {G.nnz} nnz, fp64, {world} nnz-balanced row blocks"
    return out


def halo_spmv(msp, torch, dist, dev, G, r0, r1, rank, world):
    """f4(ii): the headline's weak-scaled SpMV with a halo exchange instead of
    the x all-gather (dist.HaloSpmv); max over ranks."""
    from paper_conf_ipps_daltonbmog15_b200 import dist as mdist
    a0, a1 = int(G.rp[r0]), int(G.rp[r1])
    plan = mdist.HaloSpmv(G.rp[r0:r1 + 1] - a0, G.col[a0:a1], G.val[a0:a1], G.n, device=dev)
    plan.x_own.copy_(torch.ones(plan.own_len, dtype=plan.x_local.dtype, device=dev))
    y = torch.empty(r1 - r0, dtype=plan.x_local.dtype, device=dev)
    stream = torch.cuda.current_stream(dev)
    tm = Timer(torch, stream)
    ex, tot = [], []
    for i in range(23):
        dist.barrier()
        a = tm.ev()
        plan.exchange()
        b = tm.ev()
        msp.spmv(plan.A, plan.x_local, out=y)
        c = tm.ev()
        torch.cuda.synchronize(dev)
        if i >= 3:
            ex.append(a.elapsed_time(b))
            tot.append(a.elapsed_time(c))
    res = {}
    for k, v in (("exchange_ms", ex), ("ms", tot)):
        t = torch.tensor([float(np.mean(v))], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        res[k] = float(t.item())
    hl = torch.tensor([float(plan.halo_len)], dtype=torch.float64, device=dev)
    dist.all_reduce(hl, op=dist.ReduceOp.MAX)
    by = spmv_alg_bytes(r1 - r0, G.n, a1 - a0, 8) * world
    res.update({"GB_s": by / (res["ms"] * 1e-3) / 1e9, "max_halo_entries": int(hl.item()),
                "note": "halo exchange (one all_to_all) + local SpMV; headline uses the x all-gather"})
    return res


def msp_arm(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    import paper_conf_ipps_daltonbmog15_b200 as msp

    ops = [o for o in args.ops.split(",") if o]
    G, r0, r1 = workload(rank, world)
    m_loc = r1 - r0
    a0, a1 = int(G.rp[r0]), int(G.rp[r1])
    rp_loc = (G.rp[r0:r1 + 1] - a0).astype(np.int32)
    A = msp.CsrTensor.from_arrays(rp_loc, G.col[a0:a1], G.val[a0:a1], (m_loc, G.n), dev)
    import gen
    xg = gen.x_vector(G.n, "random", seed=1002)
    x_full = torch.as_tensor(xg, device=dev)
    x_slice = msp.dist.x_slice_of(x_full, rank, world)
    y = torch.empty(m_loc, dtype=torch.float64, device=dev)

    have = {"spmv": True, "spadd": "spadd" in ops, "spgemm": "spgemm" in ops}
    if have["spadd"]:
        T = gen.transpose(G)
        t0_, t1_ = int(T.rp[r0]), int(T.rp[r1])
        At = msp.CsrTensor.from_arrays((T.rp[r0:r1 + 1] - t0_).astype(np.int32), T.col[t0_:t1_],
                                       T.val[t0_:t1_], (m_loc, G.n), dev)
        # the one-pass SpAdd's output arrays (capacity nnz(A) + nnz(A^T)),
        # allocated once outside the timed steps
        add_col = torch.empty(A.nnz + At.nnz, dtype=torch.int32, device=dev)
        add_val = torch.empty(A.nnz + At.nnz, dtype=torch.float64, device=dev)
    Bfull = msp.dist.gather_csr_blocks(A) if (world > 1 and have["spgemm"]) else A

    stream = torch.cuda.current_stream(dev)
    tm = Timer(torch, stream)
    rec = {k: [] for k in ("spmv", "allgather", "spadd", "spgemm", "step")}
    extra = {}
    # the SpMV kernel runs on `stream`; its launch duration is taken with
    # events recorded on that same stream around each launch
    spmv_kernel_ms = []

    gemm_out = [None, None]

    def step(timed: bool):
        e0 = tm.ev()
        if world > 1:
            ea = tm.ev()
            xin = msp.dist.allgather_x(x_slice, G.n)  # NCCL all-gather of x over NVLink
            eb = tm.ev()
        else:
            xin = x_full
        sp_ev = []
        for _ in range(args.spmv_reps):
            s0 = tm.ev()
            msp.spmv(A, xin, out=y)
            s1 = tm.ev()
            sp_ev.append((s0, s1))
        ad_ev = gm_ev = None
        if have["spadd"]:
            q0 = tm.ev()
            C = msp.spadd_fused(A, At, col=add_col, val=add_val)
            q1 = tm.ev()
            ad_ev = (q0, q1)
            extra["spadd_nnz_c"] = C.nnz
        if have["spgemm"]:
            g0 = tm.ev()
            Bg = msp.dist.gather_csr_blocks(A) if world > 1 else Bfull
            P = msp.SpGemmPlan(A, Bg)
            P.setup()
            P.symbolic()
            Cg = P.numeric(col=gemm_out[0], val=gemm_out[1])
            g1 = tm.ev()
            if gemm_out[0] is None:  # C's arrays kept for the following steps (warm-up allocates)
                gemm_out[0], gemm_out[1] = Cg.col, Cg.val
            gm_ev = (g0, g1)
            extra["spgemm_nprods"] = P.nprods
            extra["spgemm_nnz_c"] = Cg.nnz
        e1 = tm.ev()
        if timed:
            torch.cuda.synchronize(dev)
            rec["step"].append(e0.elapsed_time(e1))
            lt = [a.elapsed_time(b) for a, b in sp_ev]
            spmv_kernel_ms.extend(lt)
            rec["spmv"].append(float(np.mean(lt)))
            if world > 1:
                rec["allgather"].append(ea.elapsed_time(eb))
            if ad_ev:
                rec["spadd"].append(ad_ev[0].elapsed_time(ad_ev[1]))
            if gm_ev:
                rec["spgemm"].append(gm_ev[0].elapsed_time(gm_ev[1]))

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize(dev)
    clk = ClockSampler(local)
    clk.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    L = msp.lib()
    n_launch0 = L.msp_launch_count()
    t_start = tm.ev()
    for _ in range(args.steps):
        step(True)
    t_end = tm.ev()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    clocks = clk.stop()
    n_launches = int(L.msp_launch_count() - n_launch0)
    total_ms = t_start.elapsed_time(t_end)

    def red_max(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    spmv_compute_ms = red_max(float(np.mean(rec["spmv"])))
    # N > 1: a distributed SpMV is the x all-gather (NCCL over NVLink) plus
    # the local SpMV -- each SpMV of an iterative method needs a fresh x
    spmv_ms = red_max(float(np.mean(rec["spmv"])) +
                      (float(np.mean(rec["allgather"])) if rec["allgather"] else 0.0))
    step_ms = red_max(total_ms / args.steps)
    vs = 8
    by_loc = spmv_alg_bytes(m_loc, G.n, A.nnz, vs)
    kernel_name = spmv_kernel_name(m_loc, A.nnz)  # before the table frees A
    by_all = by_loc * world if world > 1 else by_loc
    value = by_all / (spmv_ms * 1e-3) / 1e9
    peak, peak_kind = peaks()
    achieved = by_loc / (float(np.mean(spmv_kernel_ms)) * 1e-3) / 1e9
    ops_out = {"spmv": {"ms": spmv_ms, "compute_ms": spmv_compute_ms, "GB_s": value,
                        "GFLOP_s": 2 * A.nnz * world / (spmv_ms * 1e-3) / 1e9}}
    if rec["allgather"]:
        ops_out["spmv"]["allgather_ms"] = red_max(float(np.mean(rec["allgather"])))
    if rec["spadd"]:
        ms = red_max(float(np.mean(rec["spadd"])))
        ops_out["spadd"] = {"op": "A + A^T", "ms": ms, "input_nnz_per_s": 2 * A.nnz * world / (ms * 1e-3),
                            "nnz_c": extra.get("spadd_nnz_c")}
    if rec["spgemm"]:
        ms = red_max(float(np.mean(rec["spgemm"])))
        ops_out["spgemm"] = {"op": "A * A", "ms": ms,
                             "products_per_s": extra["spgemm_nprods"] * world / (ms * 1e-3),
                             "nprods": extra["spgemm_nprods"], "nnz_c": extra["spgemm_nnz_c"]}

    e2e = None
    if not args.no_e2e:
        e2e = e2e_spmv(msp, torch, G, r0, r1, dev, args)
    strong = halo = None
    if world > 1:
        strong = c5_strong(msp, torch, dist, dev, rank, world)
        halo = halo_spmv(msp, torch, dist, dev, G, r0, r1, rank, world)
    table = pred = None
    if world == 1 and not args.no_table:
        flush_buf = torch.empty(2 * L2_BYTES // 4, dtype=torch.float32, device=dev)

        def flush():
            flush_buf.fill_(1.0)
        A = At = y = Bfull = add_col = add_val = None  # noqa: F841  (free the headline workload's device memory)
        gemm_out[0] = gemm_out[1] = None
        torch.cuda.empty_cache()
        table = table_configs(msp, torch, dev, [c for c in args.table_configs.split(",") if c], peak, flush)
        pred = predictability(table)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(budget_s=10.0)
    if rank == 0:
        line = {
            "metric": METRIC,
            "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": step_ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic (seeded generators, gen/)",
            "config": {"workload": WORKLOAD_C2 if world == 1 else
                       f"3D Poisson 27-point 100x100x{100 * world} fp64, 100^3 rows per rank",
                       "ops": ",".join(k for k in ("spmv", "spadd", "spgemm") if k == "spmv" or have[k]),
                       "spmv_reps_per_step": args.spmv_reps, "parallelism": f"row blocks x{world}",
                       "l2": "inputs larger than L2 (A = 318 MB per rank > 126 MB); x (8 MB) L2-resident; "
                             "table: L2 flushed between launches for inputs < 2x L2"},
            "ops": ops_out,
            "roofline": {"bound": "hbm", "kernel": kernel_name, "achieved": achieved, "peak": peak,
                         "peak_kind": peak_kind, "unit": "GB/s", "frac": achieved / peak,
                         "alg_bytes_per_launch": by_loc, "launches_timed": len(spmv_kernel_ms),
                         **ncu_traffic(world)},
            "clocks": clocks,
            "gpu_launches": n_launches,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        if table is not None:
            line["table"] = table
            line["predictability"] = pred
        if strong is not None:
            line["c5_strong"] = strong
        if halo is not None:
            line["spmv_halo"] = halo
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()
    return 0


def e2e_spmv(msp, torch, G, r0, r1, dev, args):
    """SpMV through the public API with host buffers: pinned H2D of this
    rank's A block and x, the SpMV, D2H of y -- all inside the timed region."""
    a0, a1 = int(G.rp[r0]), int(G.rp[r1])
    h_rp = torch.from_numpy((G.rp[r0:r1 + 1] - a0).astype(np.int32)).pin_memory()
    h_col = torch.from_numpy(np.ascontiguousarray(G.col[a0:a1])).pin_memory()
    h_val = torch.from_numpy(np.ascontiguousarray(G.val[a0:a1])).pin_memory()
    import gen
    h_x = torch.from_numpy(gen.x_vector(G.n, "random", seed=1002)).pin_memory()
    m = r1 - r0
    d_rp = torch.empty_like(h_rp, device=dev)
    d_col = torch.empty_like(h_col, device=dev)
    d_val = torch.empty_like(h_val, device=dev)
    d_x = torch.empty_like(h_x, device=dev)
    h_y = torch.empty(m, dtype=torch.float64).pin_memory()
    A = msp.CsrTensor(d_rp, d_col, d_val, (m, G.n))
    y = torch.empty(m, dtype=torch.float64, device=dev)
    s = torch.cuda.current_stream(dev)

    def one():
        d_rp.copy_(h_rp, non_blocking=True)
        d_col.copy_(h_col, non_blocking=True)
        d_val.copy_(h_val, non_blocking=True)
        d_x.copy_(h_x, non_blocking=True)
        msp.spmv(A, d_x, out=y)
        h_y.copy_(y, non_blocking=True)

    for _ in range(3):
        one()
    torch.cuda.synchronize(dev)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    n = max(3, args.steps)
    e0.record(s)
    for _ in range(n):
        one()
    e1.record(s)
    torch.cuda.synchronize(dev)
    ms = e0.elapsed_time(e1) / n
    by = spmv_alg_bytes(m, G.n, a1 - a0, 8)
    h2d = sum(t.numel() * t.element_size() for t in (h_rp, h_col, h_val, h_x))
    return {"value": by / (ms * 1e-3) / 1e9, "unit": "GB/s", "ms": ms, "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": h_y.numel() * 8}


if __name__ == "__main__":
    sys.exit(main())
