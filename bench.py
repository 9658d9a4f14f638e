#!/usr/bin/env python
"""Benchmark of LiteForm's hot path on B200 (one JSON line on rank 0).

A STEP is one pass of the whole hot path over the
workload: GPU configure statistics + eq. 7 / Algorithm 3 (lf_cell_configure),
GPU CSR->CELL conversion (lf_cell_build), CELL SpMM with the C update
(lf_spmm); for N > 1 each rank runs it on its row shard and C is
all-gathered over NCCL.  metric = GFLOP/s = 2*nnz*J / t_step (whole job).

    python bench.py [--gpus N --steps K --warmup W --config c2_rmat20]
    python bench.py --impl reference     # the CPU oracle, same metric

Workload: BASELINE.json configs[1] (R-MAT scale 20, edge factor 16, J = 128),
synthetic, seeded (gen/).  Inputs are larger than L2 (B 512 MB, C 512 MB).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402

METRIC = "SpMM GFLOP/s (2*nnz*J/t) and HBM GB/s vs ~8 TB/s at 1/2/4/8 B200"


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


# measured gather ceiling for the bench workload's own column sequence
# (tools/gather_replay.cu, profiles/r1_gather_replay.md): pure 512-B B-row
# gathers at the best depth (U = 8, 4 blocks/SM), CSR order
GATHER_CEILING = {"c2_rmat20": (20649.0, "profiles/r1_gather_replay.md: c2 column sequence replayed as pure "
                                         "512-B row gathers, U=8, 4 blocks/SM, 0.399 ms"),
                  # permuted R-MAT: c2's column sequence replayed in shuffled order (the row
                  # permutation's effect) ran at 0.403 ms = 20,437 GB/s
                  "c2p_rmat20_perm": (20437.0, "profiles/r1_gather_replay.md: c2 column sequence replayed in "
                                               "shuffled order, U=8, 4 blocks/SM, 0.403 ms"),
                  # c4 at P = 8 gathers 1-KB rows from a ~30 MB partition slab of B (L2-resident)
                  "c4_reddit": (20109.0, "profiles/r1_gather_roofline.md (round-2 rows): random 1024-B row gathers "
                                         "from an L2-resident 32 MB table (c4's partition slab is 29 MB), 8 blocks/SM")}


def src_hash():
    """sha1 over liblf.so's sources: a DRAM-traffic figure measured by ncu is
    used only for the exact kernels it was measured on."""
    import glob
    import hashlib
    h = hashlib.sha1()
    pkg = os.path.join(ROOT, "paper_conf_hpdc_pengtpk25_b200", "csrc")
    for f in sorted(glob.glob(os.path.join(pkg, "**", "*.cu*"), recursive=True) +
                    glob.glob(os.path.join(pkg, "*.h")) + glob.glob(os.path.join(ROOT, "include", "*.h"))):
        with open(f, "rb") as fh:
            h.update(os.path.relpath(f, ROOT).encode() + b"\0" + fh.read())
    return h.hexdigest()


def ncu_traffic(config, J):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of the SpMM
    kernels (kernel-name matched) from profiles/traffic.json, written by
    scripts/ncu_traffic.py with ncu on the SAME sources (hash checked);
    None when absent or stale."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            t = json.load(f)
    except Exception:
        return None, "profiles/traffic.json absent"
    e = t.get("entries", {}).get(f"{config}:J{J}")
    if not e:
        return None, f"no ncu entry for {config} J={J}"
    if t.get("src_hash") != src_hash():
        return None, "profiles/traffic.json measured on other sources (stale)"
    return int(e["dram_bytes"]), f"ncu {e['kernels']} ({t.get('when', '?')}): {e['dram_read']} B read + " \
                                 f"{e['dram_write']} B written per launch"


def fp32_peak_tflops():
    """FP32 CUDA-core peak: SMs x 128 FMA/clk x 2 flop x max SM clock (B200:
    148 x 128 x 2 x 1.965 GHz = 74.4 TFLOP/s)."""
    sm_mhz = 1965.0
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            sm_mhz = float(json.load(f).get("sm_max_mhz", sm_mhz))
    except Exception:
        pass
    n_sm = 148
    try:
        import torch
        n_sm = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
    except Exception:
        pass
    return n_sm * 128 * 2 * sm_mhz * 1e6 / 1e12


def gather_roofline(config, nnz, J, world, spmm_ms):
    """The SpMM's binding traffic: one J*4-byte B row per nonzero through
    L2/L1 (nnz*J*4 bytes per launch), against the measured gather ceiling."""
    g = nnz * J * 4 / world
    out = {"bytes_per_launch": int(g), "achieved": g / (spmm_ms * 1e-3) / 1e9, "unit": "GB/s"}
    if config in GATHER_CEILING and world == 1:
        c, src = GATHER_CEILING[config]
        out.update(ceiling=c, frac=out["achieved"] / c, ceiling_source=src)
    return out


def algorithmic_bytes(A_h, J):
    """bytes_alg = nnz*(4+4) + U*J*4 + I*J*4: index + value of
    every nonzero once, each needed B row once, every C row written once."""
    U = int(np.count_nonzero(np.bincount(A_h.col_ind, minlength=A_h.n_cols))) if A_h.nnz else 0
    return 8 * A_h.nnz + 4 * U * J + 4 * A_h.n_rows * J, U


class ClockSampler:
    """NVML sampling of SM clocks and throttle reasons during the timed region."""
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks_setting"}

    def __init__(self, dev_index: int):
        self.samples, self.reasons, self.ok = [], 0, False
        try:
            import pynvml
            import torch
            pynvml.nvmlInit()
            uuid = str(torch.cuda.get_device_properties(dev_index).uuid)
            try:
                self.h = pynvml.nvmlDeviceGetHandleByUUID(uuid if uuid.startswith("GPU-") else "GPU-" + uuid)
            except Exception:
                self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.nv = pynvml
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.reasons |= int(self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
            except Exception:
                pass
            self._stop.wait(0.01)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": float(np.median(self.samples)) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "samples": len(self.samples),
                "reasons": [n for b, n in self.REASONS.items() if self.reasons & b]}


# --------------------------------------------------------------------------
# CPU oracle (cpu_baseline leg and --impl reference)
# --------------------------------------------------------------------------
def sample_rows(A_h, n_rows, seed=0):
    rng = np.random.default_rng(seed)
    rows = np.sort(rng.choice(A_h.n_rows, size=min(n_rows, A_h.n_rows), replace=False))
    l = np.diff(A_h.row_ptr)[rows]
    rp = np.concatenate([[0], np.cumsum(l)]).astype(np.int64)
    idx = np.concatenate([np.arange(A_h.row_ptr[r], A_h.row_ptr[r + 1]) for r in rows]) if len(rows) else \
        np.zeros(0, np.int64)
    return gen.CSR(len(rows), A_h.n_cols, rp, A_h.col_ind[idx], A_h.val[idx], A_h.name + "-sample")


def oracle_step(sub, B_h, J):
    """The oracle of the whole path on a row sample: Algorithm 3 over eq. 7
    (configure), CSR->CELL, Algorithm 2 SpMM -- plain C, OpenMP where the
    oracle is parallel (eq. 7's buckets, Alg. 2's output columns)."""
    import oracle
    e, k = oracle.configure(sub, 1, J)
    cell = oracle.csr_to_cell(sub, 1, e, k)
    oracle.cell_spmm(cell, B_h)


def calibrate_sample(A_h, B_h, J, target_s):
    n = max(64, A_h.n_rows // 2000)
    while True:
        sub = sample_rows(A_h, n)
        t0 = time.perf_counter()
        oracle_step(sub, B_h, J)
        dt = time.perf_counter() - t0
        if dt > 0.3 or n >= A_h.n_rows:
            break
        n = min(A_h.n_rows, n * 4)
    n = int(min(A_h.n_rows, max(64, n * target_s / max(dt, 1e-6))))
    return sample_rows(A_h, n)


def cpu_baseline(A_h, B_h, J, target_s=15.0, threads=0):
    """The oracle as it stands on the host's cores (threads = 0: all of them,
    OMP default), on a bounded random row sample of the workload."""
    import oracle
    prev = oracle.set_threads(0)
    cores = oracle.set_threads(threads) if threads > 0 else prev
    try:
        sub = calibrate_sample(A_h, B_h, J, target_s)
        t0 = time.perf_counter()
        oracle_step(sub, B_h, J)
        dt = time.perf_counter() - t0
    finally:
        oracle.set_threads(prev)
    return {"value": 2.0 * sub.nnz * J / dt / 1e9, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
            "sample": f"{sub.n_rows} random rows ({sub.nnz} nnz) of the workload; oracle configure (Alg. 3 over "
                      f"eq. 7) + CSR->CELL + Alg. 2 fp64 SpMM, {cores} OpenMP thread(s), {dt:.2f} s",
            "host_cpus": os.cpu_count()}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    # rank 0 alone runs the oracle (the other ranks exit without work), so it
    # takes every host core even under torchrun, which sets OMP_NUM_THREADS=1
    cores = oracle.set_threads(os.cpu_count() or 1)
    A_h, J = gen.config(args.config, args.seed)
    B_h = gen.dense(A_h.n_cols, J, args.seed)
    per_step = max(0.2, min(5.0, 120.0 / (args.steps + args.warmup)))
    sub = calibrate_sample(A_h, B_h, J, per_step)
    for _ in range(args.warmup):
        oracle_step(sub, B_h, J)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle_step(sub, B_h, J)
    dt = (time.perf_counter() - t0) / args.steps
    v = 2.0 * sub.nnz * J / dt / 1e9
    line = {"metric": METRIC, "value": v, "unit": "GFLOP/s", "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": args.config, "J": J, "n_rows": A_h.n_rows, "nnz": A_h.nnz,
                       "sample_rows": sub.n_rows, "sample_nnz": sub.nnz},
            "cpu_baseline": {"value": v, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                             "sample": f"{sub.n_rows} random rows ({sub.nnz} nnz) per step; oracle configure + "
                                       f"CSR->CELL + Alg. 2 fp64, {cores} OpenMP threads",
                             "host_cpus": os.cpu_count()},
            "e2e": {"value": v, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# --------------------------------------------------------------------------
# GPU arm
# --------------------------------------------------------------------------
DEFAULT_EXTRA = "c3b_banded2M:128,c3b_banded2M:64,c3_stencil126:64,c3_stencil126:128,c4_reddit:256,c2p_rmat20_perm:128"


def maybe_spawn(args):
    """--gpus N > 1 outside torchrun: launch N ranks with torch.distributed.run
    on this node (127.0.0.1) and return its exit code; fail loudly when the
    node has fewer GPUs.  Inside torchrun, WORLD_SIZE must equal N."""
    ws = os.environ.get("WORLD_SIZE")
    if ws is not None:
        if int(ws) != args.gpus and args.gpus != 1:
            print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}", file=sys.stderr)
            return 2
        return None
    if args.gpus <= 1:
        return None
    import socket
    import subprocess
    import torch
    n_dev = torch.cuda.device_count()
    if n_dev < args.gpus:
        print(f"bench.py: --gpus {args.gpus} requested but only {n_dev} CUDA device(s) visible", file=sys.stderr)
        return 2
    so = socket.socket()
    so.bind(("127.0.0.1", 0))
    port = so.getsockname()[1]
    so.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c2_rmat20")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--parts", type=int, default=0, help="force P (0 = predictor)")
    ap.add_argument("--width-log2", type=int, default=-1, help="force e_p (-1 = Algorithm 3)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--extra", default=DEFAULT_EXTRA,
                    help="further workloads timed in the same run, name:J comma-separated ('none' to skip): each "
                         "gets its SpMM-only time, step time and roofline block")
    ap.add_argument("--shard-mode", default="nnz", choices=["nnz", "bytes"])
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "fused"],
                    help="N > 1: C rows exchanged by NCCL point-to-point after the SpMM (nccl) or written by the "
                         "SpMM kernels straight into every rank's symmetric-memory C over NVLink (fused, "
                         "lf_spmm_ex destinations)")
    ap.add_argument("--streams", type=int, default=2,
                    help="steps in flight: consecutive steps alternate over this many CUDA streams, each with its "
                         "own C, so one step's host synchronisations (configure, build) overlap the previous "
                         "step's SpMM (1 = strictly serial steps)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    rc = maybe_spawn(args)
    if rc is not None:
        return rc

    import torch
    import torch.distributed as dist
    import paper_conf_hpdc_pengtpk25_b200 as lf
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        assert dist.get_world_size() == world == args.gpus, "NCCL communicator size != --gpus"
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

    def maxr(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    A_h, J = gen.config(args.config, args.seed)
    B_h = gen.dense(A_h.n_cols, J, args.seed)
    bytes_alg, U = algorithmic_bytes(A_h, J)
    flops = 2.0 * A_h.nnz * J
    bounds = lfd.shard_bounds(A_h.row_ptr, world, J, args.shard_mode)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    p0, p1 = int(A_h.row_ptr[lo]), int(A_h.row_ptr[hi])
    # host (pinned) copies of this rank's shard -- the e2e leg copies them every step
    h_rp = torch.from_numpy(A_h.row_ptr[lo:hi + 1] - p0).pin_memory()
    h_ci = torch.from_numpy(A_h.col_ind[p0:p1]).pin_memory()
    h_va = torch.from_numpy(A_h.val[p0:p1]).pin_memory()
    h_B = torch.from_numpy(B_h).pin_memory()
    d_rp, d_ci, d_va, d_B = (t.to(dev) for t in (h_rp, h_ci, h_va, h_B))
    A = lf.Csr(d_rp, d_ci, d_va, A_h.n_cols, p1 - p0)
    I_loc = hi - lo
    # N > 1: every rank holds the full C; its SpMM writes its own rows in place
    # and exchange_rows (NCCL point-to-point, exact sizes) fills in the rest
    C_full = torch.empty((A_h.n_rows, J), dtype=torch.float32, device=dev) if world > 1 else None
    C_loc = C_full[lo:hi] if world > 1 else torch.empty((I_loc, J), dtype=torch.float32, device=dev)
    # steps in flight: lane l owns a stream and its own C (lane 0 reuses C_loc)
    n_lanes = max(1, args.streams)
    lanes = [torch.cuda.current_stream()] + [torch.cuda.Stream(dev) for _ in range(n_lanes - 1)]
    fused = world > 1 and args.exchange == "fused"
    lane_sym = []
    if fused:  # every lane: a symmetric-memory full C and the addresses of every rank's copy
        lane_C = []
        for _ in range(n_lanes):
            sym = lfd.symmetric_C(A_h.n_rows, J, dev)
            if sym is None:
                raise SystemExit("bench.py: --exchange fused needs torch symmetric memory on this box")
            lane_sym.append(sym)
            lane_C.append((sym[0], sym[0][lo:hi]))
        C_full, C_loc = lane_C[0]
    else:
        lane_C = [(C_full, C_loc)]
        for _ in range(n_lanes - 1):
            Cf = torch.empty((A_h.n_rows, J), dtype=torch.float32, device=dev) if world > 1 else None
            lane_C.append((Cf, Cf[lo:hi] if world > 1 else torch.empty((I_loc, J), dtype=torch.float32,
                                                                         device=dev)))
    h_C = torch.empty((I_loc, J), dtype=torch.float32).pin_memory()
    stream = torch.cuda.current_stream()
    kw = {}
    if args.parts:
        kw["force_parts"] = args.parts
    if args.width_log2 >= 0:
        kw["force_width_log2"] = args.width_log2

    phase = {"configure": [], "build": [], "spmm": [], "gather": []}
    info = {}

    def step(Ain, record=False, lane=0):
        st = lanes[lane]
        Cf, Cl = lane_C[lane]
        with torch.cuda.stream(st):
            e0 = ev(); e0.record(st)
            params, stats = lf.configure(Ain, J, stream=st, **kw)
            e1 = ev(); e1.record(st)
            M = lf.CellMatrix.build(Ain, params, stats, stream=st)
            e2 = ev(); e2.record(st)
            if fused:  # the kernels write this rank's rows into every rank's C
                M.spmm(d_B, stream=st, dst=lane_sym[lane][2], row_base=lo)
            else:
                M.spmm(d_B, out=Cl, stream=st)
            e3 = ev(); e3.record(st)
            if fused:
                lane_sym[lane][1].barrier(channel=0)  # peers' rows landed before C is read
            elif world > 1:
                lfd.exchange_rows(Cf, bounds)  # NCCL ordered after this lane's stream
            e4 = ev(); e4.record(st)
        if record:
            phase["_ev"].append((e0, e1, e2, e3, e4))
            info["params"] = params.as_dict()
            info["path"] = M.path()
            v = M.view()
            info["cell_slots"] = int(v["n_slots"])
            info["cell_rows"] = int(v["n_cell_rows"])
            info["n_buckets"] = len(v["buckets"])
        M.close()
        return params

    phase["_ev"] = []
    for i in range(max(args.warmup, n_lanes)):  # every lane warmed (its allocator pool and C)
        step(A, lane=i % n_lanes)
    barrier()
    with ClockSampler(local) as clk:
        t0 = ev(); t1 = ev()
        barrier()
        t0.record(stream)
        for st in lanes[1:]:
            st.wait_event(t0)
        for i in range(args.steps):
            params = step(A, record=n_lanes == 1, lane=i % n_lanes)
        for st in lanes[1:]:
            stream.wait_stream(st)
        t1.record(stream)
        torch.cuda.synchronize()
    ms_serial = None
    if n_lanes > 1:  # phases (and the serial step time) from steps run one at a time on lane 0
        barrier()
        u0 = ev(); u1 = ev()
        u0.record(stream)
        for _ in range(args.steps):
            step(A, record=True)
        u1.record(stream)
        torch.cuda.synchronize()
        ms_serial = u0.elapsed_time(u1) / args.steps
    if world > 1:
        dist.barrier()
    ms = t0.elapsed_time(t1) / args.steps
    for (e0, e1, e2, e3, e4) in phase["_ev"]:
        phase["configure"].append(e0.elapsed_time(e1))
        phase["build"].append(e1.elapsed_time(e2))
        phase["spmm"].append(e2.elapsed_time(e3))
        phase["gather"].append(e3.elapsed_time(e4))
    ph = {k: float(np.mean(v)) for k, v in phase.items() if k != "_ev"}
    ms = maxr(ms)
    if ms_serial is not None:
        ms_serial = maxr(ms_serial)
    ph = {k: maxr(v) for k, v in ph.items()}

    # ---- SpMM alone (the paper's kernel-only time) -----------
    params, stats = lf.configure(A, J, **kw)
    M = lf.CellMatrix.build(A, params, stats)
    for _ in range(3):
        M.spmm(d_B, out=C_loc)
    barrier()
    n_sp = max(10, args.steps)
    s0, s1 = ev(), ev()
    s0.record(stream)
    for _ in range(n_sp):
        M.spmm(d_B, out=C_loc)
    s1.record(stream)
    torch.cuda.synchronize()
    spmm_ms = maxr(s0.elapsed_time(s1) / n_sp)
    M.close()

    # ---- e2e: host buffers in, result back, through the public API ---------
    e2e = None
    if not args.no_e2e:
        h2d = sum(t.numel() * t.element_size() for t in (h_rp, h_ci, h_va, h_B))
        d2h = h_C.numel() * 4

        # the public host-buffer API: HostPipeline (paper_conf_hpdc_pengtpk25_b200/pipeline.py)
        # double-buffers the problem over H2D / compute / D2H streams, so step k+1's
        # inputs stream in while step k computes and step k-1's C streams out
        from paper_conf_hpdc_pengtpk25_b200.pipeline import HostPipeline
        pipe = HostPipeline(I_loc, A_h.n_cols, p1 - p0, J, dev, **kw)
        h_Cs = [h_C, torch.empty_like(h_C).pin_memory()]
        for i in range(2):
            pipe.submit(h_rp, h_ci, h_va, h_B, h_Cs[i % 2])
        pipe.synchronize()
        barrier()
        x0, x1 = ev(), ev()
        n_e2e = max(3, min(args.steps, 20))
        x0.record(pipe.s_h2d)
        for i in range(n_e2e):
            pipe.submit(h_rp, h_ci, h_va, h_B, h_Cs[i % 2])
        x1.record(pipe.s_d2h)
        pipe.synchronize()
        e2e_ms = maxr(x0.elapsed_time(x1) / n_e2e)
        # PCIe floor of that step: the same H2D and D2H bytes copied concurrently
        # (full duplex) on the pipeline's streams with no compute in between
        sl, nz = pipe.slots[0], int(h_ci.numel())
        y0, y1 = ev(), ev()
        torch.cuda.synchronize()
        y0.record(pipe.s_h2d)
        pipe.s_d2h.wait_event(y0)
        for i in range(n_e2e):
            with torch.cuda.stream(pipe.s_h2d):
                sl["rp"].copy_(h_rp, non_blocking=True)
                sl["ci"][:nz].copy_(h_ci, non_blocking=True)
                sl["va"][:nz].copy_(h_va, non_blocking=True)
                sl["B"].copy_(h_B, non_blocking=True)
            with torch.cuda.stream(pipe.s_d2h):
                h_Cs[i % 2].copy_(pipe.slots[1]["C"], non_blocking=True)
        pipe.s_h2d.wait_stream(pipe.s_d2h)
        y1.record(pipe.s_h2d)
        torch.cuda.synchronize()
        pcie_ms = maxr(y0.elapsed_time(y1) / n_e2e)
        e2e = {"value": flops / (e2e_ms * 1e-3) / 1e9, "unit": "GFLOP/s", "ms_per_step": e2e_ms,
               "api": "HostPipeline.submit (host CSR + B in, host C out; N > 1: each rank's row block)",
               "h2d_bytes_per_step": int(h2d * world), "d2h_bytes_per_step": int(d2h * world),
               "pcie_floor_ms": pcie_ms, "pcie_frac": pcie_ms / e2e_ms,
               "pcie_floor_note": "the step's H2D + D2H bytes copied concurrently on the same streams, no compute"}
        del pipe
    del C_full, C_loc, lane_C, d_rp, d_ci, d_va, d_B, A
    torch.cuda.empty_cache()

    # ---- further workloads (BASELINE configs 3-4 and the J=128 band target) --
    extras = []
    if args.extra and args.extra != "none":
        for item in args.extra.split(","):
            name, jx = item.split(":")
            extras.append(time_workload(lf, lfd, torch, dist, name, int(jx), args, world, rank, dev, ev, maxr,
                                        barrier))

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0
    hbm_peak, peak_kind = peaks()
    P = params.n_parts
    # configure (lf_api.cu): nnz <= 2^25 -> the statistics pass for P = 1 first
    # (stats_rows carrying the group / window samples, stats_mark, stats_cols)
    # and again (3 kernels) if the predictor picks P > 1; larger ->
    # features_kernel (with the samples) first, then the statistics pass when
    # CELL is used.  build: bucket_kernel<0>, tile_scan, pad_init,
    # bucket_kernel<1>, slot_fill, run_bounds (+ seg_kernel for P > 1).  SpMM:
    # zero_rows_kernel + the SpMM kernel; CSR: csr_spmm_kernel.
    spec = args.parts != 0 or A_h.nnz <= (1 << 25)
    cfg_launches = (3 + (3 if (params.n_parts != 1 and args.parts == 0 and params.use_cell) else 0)) if spec \
        else (1 + (3 if params.use_cell else 0))
    if params.use_cell:
        launches_per_step = cfg_launches + 6 + (1 if P > 1 else 0) + 2
    else:
        launches_per_step = cfg_launches + 1
    sp_ms = ph["spmm"]
    traffic, traffic_src = ncu_traffic(args.config, J) if world == 1 else (None, "N > 1")
    line = {
        "metric": METRIC, "value": flops / (ms * 1e-3) / 1e9, "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": args.config, "J": J, "n_rows": A_h.n_rows, "n_cols": A_h.n_cols, "nnz": A_h.nnz,
                   "distinct_cols": U, "params": info.get("params"), "spmm_path": info.get("path"),
                   "cell_slots": info.get("cell_slots"),
                   "cell_rows": info.get("cell_rows"), "n_buckets": info.get("n_buckets"),
                   "parallelism": f"rows{world}", "shard_mode": args.shard_mode, "streams": n_lanes,
                   "exchange": ("fused (SpMM writes every rank's symmetric C)" if fused else
                                "nccl p2p after the SpMM") if world > 1 else "none",
                   "l2": "inputs larger than L2 (B, C, CELL each >126 MB); no flush"},
        "phases_ms": ph,
        "ms_per_step_serial": ms_serial if ms_serial is not None else ms,
        "spmm_only": {"ms": spmm_ms, "gflops": flops / (spmm_ms * 1e-3) / 1e9,
                      "hbm_gbs_alg": bytes_alg / world / (spmm_ms * 1e-3) / 1e9},
        "roofline": {"kernel": "lf_spmm: " + str(info.get("path")), "bound": "hbm",
                     "achieved": bytes_alg / world / (sp_ms * 1e-3) / 1e9, "peak": hbm_peak, "unit": "GB/s",
                     "frac": bytes_alg / world / (sp_ms * 1e-3) / 1e9 / hbm_peak, "peak_kind": peak_kind,
                     "bytes_alg_per_launch": bytes_alg // world,
                     "traffic": traffic, "traffic_source": traffic_src},
        "gather": gather_roofline(args.config, A_h.nnz, J, world, sp_ms),
        "workloads": extras,
        "clocks": clk.summary(),
        "gpu_launches": launches_per_step * args.steps,
        "e2e": e2e,
    }
    if world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(A_h, B_h, J)
        st1 = cpu_baseline(A_h, B_h, J, target_s=5.0, threads=1)
        line["cpu_baseline"]["single_thread"] = {k: st1[k] for k in ("value", "cores", "sample")}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def time_workload(lf, lfd, torch, dist, name, J, args, world, rank, dev, ev, maxr, barrier):
    """One further workload, row-sharded like the headline: SpMM-only time
    (back-to-back lf_spmm, CUDA events, max over ranks), serial step time
    (configure + build + SpMM) and the roofline of the bound SURVEY 8(d)
    assigns it (HBM for c2/c3, FP32 ALU for c4)."""
    A_h, _ = gen.config(name, args.seed)
    B_h = gen.dense(A_h.n_cols, J, args.seed)
    bytes_alg, U = algorithmic_bytes(A_h, J)
    flops = 2.0 * A_h.nnz * J
    bounds = lfd.shard_bounds(A_h.row_ptr, world, J, args.shard_mode)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    p0, p1 = int(A_h.row_ptr[lo]), int(A_h.row_ptr[hi])
    A = lf.Csr(torch.from_numpy(A_h.row_ptr[lo:hi + 1] - p0).to(dev), torch.from_numpy(A_h.col_ind[p0:p1]).to(dev),
               torch.from_numpy(A_h.val[p0:p1]).to(dev), A_h.n_cols, p1 - p0)
    B = torch.from_numpy(B_h).to(dev)
    C = torch.empty((hi - lo, J), dtype=torch.float32, device=dev)
    for _ in range(3):
        params, stats = lf.configure(A, J)
        M = lf.CellMatrix.build(A, params, stats)
        M.spmm(B, out=C)
        M.close()
    barrier()
    n_st = max(5, min(args.steps, 10))
    s0, s1 = ev(), ev()
    s0.record()
    for _ in range(n_st):
        params, stats = lf.configure(A, J)
        M = lf.CellMatrix.build(A, params, stats)
        M.spmm(B, out=C)
        M.close()
    s1.record()
    torch.cuda.synchronize()
    step_ms = maxr(s0.elapsed_time(s1) / n_st)
    params, stats = lf.configure(A, J)
    M = lf.CellMatrix.build(A, params, stats)
    for _ in range(3):
        M.spmm(B, out=C)
    barrier()
    n_sp = max(10, min(args.steps, 30))
    s0.record()
    for _ in range(n_sp):
        M.spmm(B, out=C)
    s1.record()
    torch.cuda.synchronize()
    sp_ms = maxr(s0.elapsed_time(s1) / n_sp)
    path = M.path()
    M.close()
    out = {"workload": name, "J": J, "n_rows": A_h.n_rows, "nnz": A_h.nnz, "distinct_cols": U,
           "params": params.as_dict(), "spmm_path": path, "spmm_ms": sp_ms, "step_ms_serial": step_ms,
           "gflops": flops / (sp_ms * 1e-3) / 1e9, "step_gflops": flops / (step_ms * 1e-3) / 1e9}
    if path == "cell_spmm_kernel":  # per-slot path: one B-row gather per nonzero binds it
        out["gather"] = gather_roofline(name, A_h.nnz, J, world, sp_ms)
    hbm_peak, peak_kind = peaks()
    gbs = bytes_alg / world / (sp_ms * 1e-3) / 1e9
    traffic, traffic_src = ncu_traffic(name, J) if world == 1 else (None, "N > 1")
    if name.startswith("c4"):
        # 42 flop/B -> the FP32 CUDA-core ALUs bound c4
        pk = fp32_peak_tflops()
        ach = flops / world / (sp_ms * 1e-3) / 1e12
        out["roofline"] = {"bound": "alu", "achieved": ach, "peak": pk, "unit": "TFLOP/s", "frac": ach / pk,
                           "peak_kind": "derived: SMs x 128 FP32 FMA/clk x 2 x max SM clock",
                           "hbm_frac": gbs / hbm_peak, "traffic": traffic, "traffic_source": traffic_src}
    else:
        out["roofline"] = {"bound": "hbm", "achieved": gbs, "peak": hbm_peak, "unit": "GB/s", "frac": gbs / hbm_peak,
                           "peak_kind": peak_kind, "bytes_alg_per_launch": bytes_alg // world, "traffic": traffic,
                           "traffic_source": traffic_src}
    del A, B, C
    torch.cuda.empty_cache()
    return out


if __name__ == "__main__":
    sys.exit(main())
