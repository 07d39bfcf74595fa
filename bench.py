#!/usr/bin/env python
"""Benchmark of the merge-path hot path on B200 (BASELINE.json metric).

A step = one pass of the whole hot path over the C2 workload (BJ:8,
configs[1], the config BASELINE.json's metric is quoted on): SpMV y = A x,
SpAdd C = A + A^T and SpGEMM C = A A (setup + symbolic + numeric) on the
3-D 27-point Poisson matrix 100^3 in fp64.  `value` is the SpMV achieved
GB/s (algorithmic bytes / time); per-op numbers (SpMV GFLOP/s,
SpAdd input nnz/s, SpGEMM products/s) are reported beside it.

Multi-GPU (torchrun, N > 1): weak scaling -- rank r owns a 100^3 slab of a
100 x 100 x (100 N) Poisson grid (nnz-balanced row blocks), x is all-gathered
over NCCL before the local SpMV and B = A's row blocks are all-gathered
before the local SpGEMM.  Timing is the max over ranks.

--impl reference times the CPU oracle (the plain C reference written from the
paper) on the host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
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


# --------------------------------------------------------------- workload

def workload(rank: int, world: int):
    """C2 (world == 1) or this rank's 100^3 slab of a 100x100x(100*world) grid."""
    import gen
    if world == 1:
        A = gen.config("C2", "random")
        return A, A, 0, A.m
    G = gen.poisson3d_27pt(100, 100, 100 * world)
    G = G.with_values(gen.matrices.random_values(G.nnz, 1002))
    from paper_conf_ipps_daltonbmog15_b200 import row_split  # libmsp host helper
    starts = row_split(G.rp, world)
    return G, None, int(starts[rank]), int(starts[rank + 1])


def ncu_traffic(world):
    """DRAM bytes per launch of the SpMV kernel on C2 from the committed ncu
    --set full capture (dram__bytes_read.sum + dram__bytes_write.sum)."""
    try:
        d = json.loads((ROOT / "profiles" / "r1b_ncu_full_summary.json").read_text())
        k = d["spmv_merge_kernel C2 (row-aligned, K=27)"]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rd = float(k["dram__bytes_read.sum"][0]) * scale[k["dram__bytes_read.sum"][1]]
        wr = float(k["dram__bytes_write.sum"][0]) * scale[k["dram__bytes_write.sum"][1]]
        if world != 1:
            return {"traffic": None, "traffic_source": "ncu capture is of the 1-GPU C2 launch"}
        return {"traffic": rd + wr, "traffic_source": "profiles/r1b_ncu_full_summary.json (ncu --set full, C2 launch)"}
    except Exception as e:  # noqa: BLE001
        return {"traffic": None, "traffic_source": f"unavailable: {e}"}


def spmv_alg_bytes(m, n, nnz, vsize):
    """4 (col) + s (val) per nonzero, 4 (offset) + s (y) per row,
    s (x) per column read once; plus the final row offset."""
    return nnz * (4 + vsize) + m * (4 + vsize) + 4 + n * vsize


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
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return reference_arm(args)
    return msp_arm(args)


# --------------------------------------------------------------- reference arm

def reference_arm(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    res = cpu_baseline(budget_s=max(2.0, 6.0 * (args.steps + args.warmup) / 20))
    line = {"impl": "reference", "metric": METRIC, "value": res["value"],
            "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded generators, gen/)",
            "config": {"workload": WORKLOAD_C2, "kernel": "CPU oracle (scalar CSR, P:364-370), host cores"},
            "cpu_baseline": res, "e2e": {"value": res["value"], "unit": "GB/s", "h2d_bytes_per_step": 0,
                                          "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


def cpu_baseline(budget_s=10.0):
    """The oracle as it stands (test infrastructure) on this host, bounded."""
    import gen
    import oracle
    A = gen.config("C2", "random")
    x = gen.x_vector(A.n, "random", seed=1002)
    oracle.spmv(A, x)  # warm
    t0 = time.perf_counter()
    reps = 0
    while time.perf_counter() - t0 < budget_s:
        oracle.spmv(A, x)
        reps += 1
    dt = (time.perf_counter() - t0) / reps
    by = spmv_alg_bytes(A.m, A.n, A.nnz, 8)
    return {"value": by / dt / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
            "sample": f"full C2 SpMV x{reps} in {reps * dt:.1f}s (single-threaded C oracle)",
            "ms_per_spmv": dt * 1e3}


# --------------------------------------------------------------- msp arm

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
    G, _, r0, r1 = workload(rank, world)
    m_loc = r1 - r0
    a0, a1 = int(G.rp[r0]), int(G.rp[r1])
    rp_loc = (G.rp[r0:r1 + 1] - a0).astype(np.int32)
    A = msp.CsrTensor.from_arrays(rp_loc, G.col[a0:a1], G.val[a0:a1], (m_loc, G.n), dev)
    import gen
    xg = gen.x_vector(G.n, "random", seed=1002)
    x_full = torch.as_tensor(xg, device=dev)
    # x slice owned by this rank (equal slices, padded) for the all-gather
    x_slice = msp.dist.x_slice_of(x_full, rank, world)
    y = torch.empty(m_loc, dtype=torch.float64, device=dev)

    have = {"spmv": True, "spadd": "spadd" in ops, "spgemm": "spgemm" in ops}
    # SpAdd workload: A + A^T on the local rows (A^T rows = transpose of the
    # full matrix restricted to this rank's rows)
    if have["spadd"]:
        T = gen.transpose(G)
        t0_, t1_ = int(T.rp[r0]), int(T.rp[r1])
        At = msp.CsrTensor.from_arrays((T.rp[r0:r1 + 1] - t0_).astype(np.int32), T.col[t0_:t1_],
                                       T.val[t0_:t1_], (m_loc, G.n), dev)
        try:
            msp.SpAddPlan(A, At).symbolic()
        except msp.MspError as e:
            if e.status != 9:
                raise
            have["spadd"] = False
    if have["spgemm"]:
        Bfull = msp.dist.gather_csr_blocks(A) if world > 1 else A
        try:
            msp.SpGemmPlan(A, Bfull).setup()
        except msp.MspError as e:
            if e.status != 9:
                raise
            have["spgemm"] = False

    stream = torch.cuda.current_stream(dev)
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    rec = {k: [] for k in ("spmv", "allgather", "spadd", "spgemm", "step")}
    extra = {}

    def step(timed: bool):
        e0 = ev(); e0.record(stream)
        # SpMV (x all-gathered over NCCL when distributed)
        if world > 1:
            ea = ev(); ea.record(stream)
            xin = msp.dist.allgather_x(x_slice, G.n)  # NCCL all-gather of x over NVLink
            eb = ev(); eb.record(stream)
        else:
            xin = x_full
        sp_ev = []
        for _ in range(args.spmv_reps):
            s0 = ev(); s0.record(stream)
            msp.spmv(A, xin, out=y)
            s1 = ev(); s1.record(stream)
            sp_ev.append((s0, s1))
        ad_ev = gm_ev = None
        if have["spadd"]:
            q0 = ev(); q0.record(stream)
            C = msp.spadd(A, At)
            q1 = ev(); q1.record(stream)
            ad_ev = (q0, q1)
            extra["spadd_nnz_c"] = C.nnz
        if have["spgemm"]:
            g0 = ev(); g0.record(stream)
            # multi-GPU: replicate B's row blocks (the SpGEMM exchange step)
            Bg = msp.dist.gather_csr_blocks(A) if world > 1 else Bfull
            P = msp.SpGemmPlan(A, Bg)
            P.setup()
            P.symbolic()
            Cg = P.numeric()
            g1 = ev(); g1.record(stream)
            gm_ev = (g0, g1)
            extra["spgemm_nprods"] = P.nprods
            extra["spgemm_nnz_c"] = Cg.nnz
        e1 = ev(); e1.record(stream)
        if timed:
            torch.cuda.synchronize(dev)
            rec["step"].append(e0.elapsed_time(e1))
            rec["spmv"].append(float(np.mean([a.elapsed_time(b) for a, b in sp_ev])))
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
    t_start = ev(); t_end = ev()
    t_start.record(stream)
    for _ in range(args.steps):
        step(True)
    t_end.record(stream)
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
    by_all = by_loc * world if world > 1 else by_loc
    # GB/s of the whole job: all ranks' algorithmic bytes over the slowest rank
    value = by_all / (spmv_ms * 1e-3) / 1e9
    peak, peak_kind = peaks()
    achieved = by_loc / (float(np.mean(rec["spmv"])) * 1e-3) / 1e9
    ops_out = {"spmv": {"ms": spmv_ms, "compute_ms": spmv_compute_ms, "GB_s": value,
                        "GFLOP_s": 2 * A.nnz * world / (spmv_ms * 1e-3) / 1e9}}
    if rec["allgather"]:
        ops_out["spmv"]["allgather_ms"] = red_max(float(np.mean(rec["allgather"])))
    if rec["spadd"]:
        ms = red_max(float(np.mean(rec["spadd"])))
        ops_out["spadd"] = {"ms": ms, "input_nnz_per_s": 2 * A.nnz * world / (ms * 1e-3),
                            "nnz_c": extra.get("spadd_nnz_c")}
    if rec["spgemm"]:
        ms = red_max(float(np.mean(rec["spgemm"])))
        ops_out["spgemm"] = {"ms": ms, "products_per_s": extra["spgemm_nprods"] * world / (ms * 1e-3),
                             "nprods": extra["spgemm_nprods"], "nnz_c": extra["spgemm_nnz_c"]}

    e2e = None
    if not args.no_e2e:
        e2e = e2e_spmv(msp, torch, G, r0, r1, dev, args)
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
                       "l2": "inputs larger than L2 (A = 318 MB per rank > 126 MB); x (8 MB) L2-resident"},
            "ops": ops_out,
            "roofline": {"bound": "hbm", "kernel": "spmv_merge_kernel", "achieved": achieved, "peak": peak,
                         "peak_kind": peak_kind, "unit": "GB/s", "frac": achieved / peak,
                         "alg_bytes_per_launch": by_loc, **ncu_traffic(world)},
            "clocks": clocks,
            "gpu_launches": n_launches,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
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
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
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
