#!/usr/bin/env python
"""Benchmark: SpGEMM GFLOP/s (2 * intermediate products / time) for C = A.A on the
webbase-1M-shaped synthetic matrix (BASELINE.json metric, configs[1]) on N GPUs.

One step = the whole hot path on one input: row analysis + classification + symbolic
(incl. the nnz(C) readback) + numeric with fused compaction.  Inputs are
resident in HBM before timing; L2 is flushed (256 MiB memset) between timed steps.  N > 1:
rows are flop-partitioned across ranks (a5), B resident on every rank (replicated with an NCCL
broadcast before timing), each rank times its block, the max over ranks is the step time and
`value` is 2 * F_total / that time (strong scaling: total work fixed).  `python bench.py
--gpus N` outside torchrun re-launches itself under torch.distributed.run with N ranks.

The roofline object is the numeric phase's HBM roofline on SURVEY.md §8(d)'s compulsory bytes
(A + B + C); the plan the symbolic phase leaves (4 bytes per product) is reported next to it as
`plan_bytes` / `with_plan_frac`, not counted as algorithmic.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config webbase1m] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "SpGEMM GFLOP/s (2·flops/time) C=A·A webbase-1M-shaped, 1/2/4/8 B200"
UNIT = "GFLOP/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=100)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--config", default="webbase1m")
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-flush", action="store_true", help="do not flush L2 between steps")
    p.add_argument("--profile", action="store_true", help="short run for ncu (no baselines, no clocks)")
    p.add_argument("--opt", action="append", default=[], help="library option name=value")
    p.add_argument("--out", default=None, help="also append the JSON line to this file")
    p.add_argument("--sim-ranks-on-one-gpu", dest="virtual", action="store_true",
                   help="N>1 on one GPU for testing: gloo process group, virtual-rank handles (no NCCL)")
    return p.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def relaunch_if_needed(args) -> bool:
    """--gpus N (N > 1) outside torchrun: run this script under torch.distributed.run with N ranks.
    Returns True if this process only supervised the child launcher."""
    if "WORLD_SIZE" in os.environ:
        ws = int(os.environ["WORLD_SIZE"])
        if ws != args.gpus and not args.virtual:
            sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}")
        return False
    if args.gpus <= 1:
        return False
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except (OSError, subprocess.TimeoutExpired):
        pass
    return "unknown"


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as fh:
            d = json.load(fh)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 50 ms in the background."""
    FIELDS = ["clocks.sm", "clocks.max.sm", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap", "power.draw"]

    def __init__(self, gpu_index: int):
        self.samples = []
        self.proc = None
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(gpu_index), f"--query-gpu={','.join(self.FIELDS)}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except (FileNotFoundError, OSError):
            return
        self.t = threading.Thread(target=self._read, daemon=True)
        self.t.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 6:
                self.samples.append((time.time(), parts))

    def wait_ready(self, timeout=5.0):
        t0 = time.time()
        while self.proc and not self.samples and time.time() - t0 < timeout:
            time.sleep(0.05)

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self, t0, t1):
        if not self.proc:
            return None
        win = [p for (t, p) in self.samples if t0 <= t <= t1]
        if not win:  # timed region shorter than one sample period: take the nearest samples
            win = [p for (t, p) in sorted(self.samples, key=lambda s: min(abs(s[0] - t0), abs(s[0] - t1)))[:3]]
        if not win:
            return None

        def num(x):
            try:
                return float(x)
            except ValueError:
                return None
        sm = [num(p[0]) for p in win if num(p[0]) is not None]
        mx = [num(p[1]) for p in win if num(p[1]) is not None]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for p in win for k in range(4) if p[2 + k].lower().startswith("active")})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(win)}


def csr_bytes(nrows, nnz, vb, rp_bytes=4):
    return rp_bytes * (nrows + 1) + (4 + vb) * nnz


def oracle_sample(A, B, target_s: float, nthreads: int):
    """Time the oracle (as it stands) on a leading row range sized for ~target_s seconds."""
    import oracle
    f = oracle.row_flops(A, B)
    pf = np.concatenate([[0], np.cumsum(f)])
    F = int(pf[-1])
    # calibrate on ~0.3% of the products
    r_cal = int(np.searchsorted(pf, max(1, F // 300)))
    r_cal = max(1, min(A.nrows, r_cal))
    t0 = time.perf_counter()
    oracle.spgemm(A, B, 0, r_cal, nthreads=nthreads, with_abs=False)
    dt = max(time.perf_counter() - t0, 1e-3)
    rate = max(pf[r_cal], 1) / dt
    want = min(F, int(rate * target_s))
    r1 = int(np.searchsorted(pf, want))
    r1 = max(1, min(A.nrows, r1))
    return r1, int(pf[r1]), F


def run_reference(args):
    ws, rank, local = dist_env()
    if rank != 0:
        return
    import workloads as W
    import oracle
    A, B = W.make(args.config)
    T = os.cpu_count() or 1
    budget = 150.0 / max(1, args.steps + args.warmup)
    r1, Fs, F = oracle_sample(A, B, budget, T)
    times = []
    for s in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.spgemm(A, B, 0, r1, nthreads=T, with_abs=False)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            times.append(dt)
    t = float(np.mean(times))
    val = 2.0 * Fs / t / 1e9
    sample = f"rows [0, {r1}) of {args.config} ({Fs} of {F} products, {100.0 * Fs / F:.2f}%), {T} threads"
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64" if np.dtype(A.vals.dtype) == np.float64 else "f32",
            "data": "synthetic", "config": {"workload": args.config},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": T, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line, args)


def emit(line, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as fh:
            fh.write(s + "\n")


def slice_rows(A, r0, r1):
    import workloads as W
    rp = A.row_ptr[r0:r1 + 1]
    s, e = int(rp[0]), int(rp[-1])
    return W.CSR(r1 - r0, A.ncols, (rp - s).astype(np.int32), A.col_idx[s:e], A.vals[s:e])


def pinned(a):
    import torch
    t = torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    return t.numpy()


def run_ours(args):
    import torch
    import torch.distributed as dist
    import workloads as W
    import paper_conf_ipps_ramamoorthybsk15_b200 as spg

    ws, rank, local = dist_env()
    if args.virtual:
        local = 0
    torch.cuda.set_device(local)
    if ws > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if args.virtual:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cdev = torch.device("cpu") if args.virtual else torch.device("cuda", local)  # collective tensors
    dev = torch.device("cuda", local)
    A, B = W.make(args.config)
    same = B is A
    vdt = torch.float64 if np.dtype(A.vals.dtype) == np.float64 else torch.float32
    vb = 8 if vdt == torch.float64 else 4
    dA = spg.DeviceCSR.from_host(A, dev)
    dB = dA if same else spg.DeviceCSR.from_host(B, dev)
    stream = torch.cuda.current_stream()
    if ws > 1 and args.virtual:
        h = spg.spg_create_dist(local, stream, vdt, None, rank, ws)   # partitioned rows, no communicator
    elif ws > 1:
        obj = [spg.spg_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        h = spg.spg_create_dist(local, stream, vdt, obj[0], rank, ws)
        spg.spg_broadcast_csr(h, dB, 0)          # B replicated from rank 0 (outside timing)
        torch.cuda.synchronize()
    else:
        h = spg.spg_create(local, stream, vdt)
    spg.spg_set_option(h, "timing", 1)
    for kv in args.opt:
        k, v = kv.split("=")
        spg.spg_set_option(h, k, int(v))
    rp = torch.empty(A.nrows + 1, dtype=torch.int64, device=dev)
    nnz, rb, re = spg.spg_spgemm_symbolic(h, dA, dB, rp)
    col = torch.empty(max(nnz, 1), dtype=torch.int32, device=dev)
    val = torch.empty(max(nnz, 1), dtype=vdt, device=dev)
    spg.spg_spgemm_numeric(h, dA, dB, rp, col, val)
    torch.cuda.synchronize()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def step():
        spg.spg_spgemm_symbolic(h, dA, dB, rp)
        spg.spg_spgemm_numeric(h, dA, dB, rp, col, val)

    for _ in range(args.warmup):
        if not args.no_flush:
            flush.zero_()
        step()
    torch.cuda.synchronize()
    sampler = None if args.profile else ClockSampler(local)
    if sampler:
        sampler.wait_ready()
    K = args.steps
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(K)]
    path_ms = np.zeros(3)  # symbolic: analysis+classify, light tiles, heavy rows
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_wall0 = time.time()
    for s in range(K):
        if not args.no_flush:
            flush.zero_()
        e0, e1, e2 = ev[s]
        e0.record(stream)
        spg.spg_spgemm_symbolic(h, dA, dB, rp)
        e1.record(stream)
        spg.spg_spgemm_numeric(h, dA, dB, rp, col, val)
        e2.record(stream)
        sts = spg.spg_get_stats(h)
        path_ms += np.array([sts["ms_analysis"], sts["ms_light"], sts["ms_heavy"]])
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    t_wall1 = time.time()
    if sampler:
        sampler.stop()
    sym = np.array([ev[s][0].elapsed_time(ev[s][1]) for s in range(K)])
    num = np.array([ev[s][1].elapsed_time(ev[s][2]) for s in range(K)])
    tot_ms = float(sym.sum() + num.sum())
    st = spg.spg_get_stats(h)
    if ws > 1:
        t = torch.tensor([tot_ms], dtype=torch.float64, device=cdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tot_ms = float(t.item())
    ms_step = tot_ms / K
    F_total = int(st["flops_total"])
    value = 2.0 * F_total / (ms_step * 1e-3) / 1e9

    # roofline of the numeric phase (k_numeric, one launch per step): SURVEY.md §8(d)'s compulsory
    # bytes A + B + C of this rank's rows; the plan read is this design's overhead, reported apart
    nnzA_loc = int(A.row_ptr[re]) - int(A.row_ptr[rb])
    abc_bytes = (csr_bytes(re - rb, nnzA_loc, vb) + csr_bytes(B.nrows, B.nnz, vb)
                 + csr_bytes(re - rb, nnz, vb, rp_bytes=8))
    plan_bytes = int(st["plan_bytes"])
    num_ms = float(np.mean(num))
    peak, peak_src = load_peaks()
    achieved = abc_bytes / (num_ms * 1e-3) / 1e9
    traffic = None
    tpath = os.path.join(ROOT, "profiles", f"traffic_{args.config}.json")
    if os.path.exists(tpath):
        with open(tpath) as fh:
            traffic = json.load(fh).get("numeric_dram_bytes_per_launch")

    # e2e through the host-pointer C ABI (H2D of inputs + D2H of C inside the timed region)
    e2e = None
    if not args.no_e2e and not args.profile:
        s0, s1 = (rb, re)
        Ah = A if ws == 1 else slice_rows(A, s0, s1)
        Ap = W.CSR(Ah.nrows, Ah.ncols, pinned(Ah.row_ptr), pinned(Ah.col_idx), pinned(Ah.vals))
        Bp = Ap if (same and ws == 1) else W.CSR(B.nrows, B.ncols, pinned(B.row_ptr), pinned(B.col_idx),
                                                 pinned(B.vals))
        h2 = spg.spg_create(local, stream, vdt)
        rph = pinned(np.empty(Ah.nrows + 1, np.int64))
        n2 = spg.spg_spgemm_host_symbolic(h2, Ap, Bp, rph)
        colh = pinned(np.empty(max(n2, 1), np.int32))
        valh = pinned(np.empty(max(n2, 1), np.float64 if vb == 8 else np.float32))
        spg.spg_spgemm_host_numeric(h2, colh, valh)
        E = min(K, 5)
        times = []
        for s in range(E + 1):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            spg.spg_spgemm_host_symbolic(h2, Ap, Bp, rph)
            spg.spg_spgemm_host_numeric(h2, colh, valh)
            times.append(time.perf_counter() - t0)
        spg.spg_spgemm_free(h2)
        e_ms = float(np.mean(times[1:])) * 1e3
        if ws > 1:
            t = torch.tensor([e_ms], dtype=torch.float64, device=cdev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_ms = float(t.item())
        h2d = csr_bytes(Ah.nrows, Ah.nnz, vb) + (0 if Bp is Ap else csr_bytes(B.nrows, B.nnz, vb))
        d2h = 8 * (Ah.nrows + 1) + (4 + vb) * n2
        e2e = {"value": 2.0 * F_total / (e_ms * 1e-3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": e_ms,
               "timer": "host wall clock around the synchronous host-pointer API calls"}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline and not args.profile:
        T = os.cpu_count() or 1
        import oracle
        r1, Fs, F = oracle_sample(A, B, 12.0, T)
        t0 = time.perf_counter()
        oracle.spgemm(A, B, 0, r1, nthreads=T, with_abs=False)
        dt = time.perf_counter() - t0
        s1, Fs1, _ = oracle_sample(A, B, 8.0, 1)  # single-thread leg
        t1 = time.perf_counter()
        oracle.spgemm(A, B, 0, s1, nthreads=1, with_abs=False)
        dt1 = time.perf_counter() - t1
        cpu = {"value": 2.0 * Fs / dt / 1e9, "unit": UNIT, "cores": T, "kind": "oracle",
               "cpu_model": cpu_model(),
               "sample": f"rows [0, {r1}) of {args.config}: {Fs} of {F} products ({100.0 * Fs / F:.1f}%), "
                         f"{dt:.1f} s on {T} threads (std::map Gustavson, as it stands)",
               "single_thread": {"value": 2.0 * Fs1 / dt1 / 1e9, "unit": UNIT, "cores": 1,
                                 "sample": f"rows [0, {s1}): {Fs1} products, {dt1:.1f} s on 1 thread"}}

    clocks = sampler.summary(t_wall0, t_wall1) if sampler else None
    stl = st
    launches = (st["launches_symbolic"] + st["launches_numeric"]) * K
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws, "steps": K, "warmup": args.warmup,
            "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64" if vb == 8 else "f32", "data": "synthetic",
            "config": {"workload": args.config, "rows": A.nrows, "nnzA": A.nnz, "nnzB": B.nnz, "flops": F_total,
                       "nnzC": int(st["nnz_c"]) if ws == 1 else None,
                       "l2": "flushed between timed steps (256 MiB memset)" if not args.no_flush else "not flushed",
                       "parallelism": (f"rows flop-partitioned over {ws} GPU(s)" + (" (virtual ranks on one GPU)"
                                       if args.virtual else "")) if ws > 1 else "1 GPU",
                       "options": args.opt},
            "ms_per_step_median": float(np.median(sym + num)), "ms_per_step_min": float(np.min(sym + num)),
            "phases": {"symbolic_ms": float(np.mean(sym)), "numeric_ms": num_ms,
                       "symbolic_ms_median": float(np.median(sym)), "numeric_ms_median": float(np.median(num)),
                       "numeric_ms_min": float(np.min(num)),
                       "numeric_gflops": 2.0 * int(st["flops"]) / (num_ms * 1e-3) / 1e9,
                       "symbolic_path_ms": dict(zip(["analysis", "light", "heavy"], (path_ms / K).round(4).tolist())),
                       "tiles": int(st["tiles"]), "heavy_rows": int(st["heavy_rows"]), "dup_products": int(st["dup_products"]),
                       "plan_bytes": int(st["plan_bytes"]),
                       "class_rows": dict(zip(spg.CLASS_NAMES, stl["class_rows"])),
                       "class_flops": dict(zip(spg.CLASS_NAMES, stl["class_flops"]))},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                         "kernel": "k_numeric (numeric phase: one launch per step)",
                         "algorithmic_bytes": int(abc_bytes), "bytes_def": "A + B + C (SURVEY.md 8d)",
                         "plan_bytes": plan_bytes,
                         "with_plan_frac": (abc_bytes + plan_bytes) / (num_ms * 1e-3) / 1e9 / peak},
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches), "clocks": clocks,
        }
        emit(line, args)
    spg.spg_spgemm_free(h)
    if ws > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    relaunch_if_needed(args)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
