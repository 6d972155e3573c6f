#!/usr/bin/env python
"""bench.py — the driver's benchmark contract for the CPU-Free Jacobi hot path.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--impl ours|reference]

One "step" is one pass of the whole hot path over the BASELINE.json workload: one
``jacobi_run(iters)`` call — ONE persistent kernel per GPU running every iteration with the
halo exchange, flags and grid barriers inside.  At N = 1 the
workload is BASELINE.json configs[1] (C2: 2D 5-point 16384x16384 fp64, 1000 iterations).
``value`` = interior cells x iterations x steps / max-over-ranks device time (CUDA events on the
launch stream around each launch), in Gcell-updates/s.  Inputs (2 GiB per buffer) are larger
than the 126 MB L2, so no flush is needed between steps.

N GPUs: under torchrun (WORLD_SIZE > 1) one rank per GPU, slabs linked by CUDA IPC; without
torchrun ``--gpus N`` drives N GPUs from one process (jacobi_create(ngpus=N): UVA peer stores
after cudaDeviceEnablePeerAccess) and exits with an error (JACOBI_ENODEV) if fewer are visible.
C2/C3 keep the grid (strong scaling), C4 grows it to 512x512x(512N) (weak scaling).

Extra keys: ``roofline`` (the persistent kernel vs the measured HBM copy bandwidth, per GPU;
µs/iteration for the L2-resident latency configs C1/C5), ``cpu_baseline`` (the CPU oracle on
this host's cores, bounded sample), ``e2e`` (the same metric through the C ABI with pinned host
buffers: scatter + run + gather per step), ``cpu_controlled`` (the per-iteration-launch
baselines), ``clocks``; at N > 1 ``halo_us`` (per-iteration time of
no-compute runs, CPU-Free vs the CPU-controlled baselines), ``halo_traffic`` (halo
bytes per iteration and GB/s vs NVLink's 900 GB/s) and ``halo_spans_*`` (in-kernel %globaltimer
wait -> flag -> signal spans of the boundary blocks, jacobi_halo_trace).  ``parity``: where
tests/golden holds the oracle's digest of the workload (C1, C2, C3 at their lengths), the SHA-256
of the whole field the e2e step produced on the N GPUs, compared with it.

``--impl reference``: there is no reference implementation to install (PAPER.md only), so
the reference arm is the CPU oracle timed on this host.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

with open(os.path.join(ROOT, "BASELINE.json")) as _f:
    _BJ = json.load(_f)
METRIC = _BJ["metric"]
UNIT = "Gcell-updates/s"

# Workloads of BASELINE.json "configs".  shape = (nz, ny, nx) incl. boundary.
CONFIGS = {
    "c1": dict(shape=(1, 256, 256), iters=1000, scaling="strong",
               workload="C1: 2D 5-point Jacobi 256x256 fp64, Dirichlet boundary, 1000 iterations"),
    "c2": dict(shape=(1, 16384, 16384), iters=1000, scaling="strong",
               workload="C2: 2D 5-point Jacobi 16384x16384 fp64, 1000 iterations, row-slab decomposition"),
    "c3": dict(shape=(512, 512, 512), iters=1000, scaling="strong",
               workload="C3: 3D 7-point Jacobi 512^3 fp64, 1000 iterations, z-slab decomposition"),
    "c4": dict(shape=None, iters=1000, scaling="weak",
               workload="C4: 3D 7-point Jacobi weak scaling 512x512x(512*P) fp64, 1000 iterations"),
    "c5a": dict(shape=(128, 128, 128), iters=1000, scaling="strong",
                workload="C5a: 3D 7-point Jacobi 128^3 fp64 latency sweep, 1000 iterations"),
    "c5b": dict(shape=(1, 1024, 1024), iters=1000, scaling="strong",
                workload="C5b: 2D 5-point Jacobi 1024x1024 fp64 latency sweep, 1000 iterations"),
}
L2_BYTES = 126 * 1024 * 1024


def interior_cells(shape):
    nz, ny, nx = shape
    return (nx - 2) * (ny - 2) * (max(nz - 2, 1) if nz > 1 else 1)


def measured_hbm():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if not self.proc:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for n, v in zip(names, parts[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def torch_device_count() -> int:
    import torch
    return torch.cuda.device_count()


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def oracle_sample(shape, iters_sample, seed=0x5C24, field=None):
    """Time the CPU oracle (as it stands) on this host's cores; returns (Gcell/s, seconds, cores)."""
    import oracle
    from jacobi_inputs import u12
    if field is None:
        field = u12(shape if shape[0] > 1 else shape[1:], seed)
    cores = os.cpu_count() or 1
    t0 = time.perf_counter()
    oracle.jacobi(field, iters_sample, cores)
    dt = time.perf_counter() - t0
    return interior_cells(shape) * iters_sample / dt / 1e9, dt, cores


def ncu_traffic(config: str, iters: int):
    """dram bytes per launch from the committed ncu --set full summary of this config, if any."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        e = d[config]
        return e["dram_bytes_per_iter"] * iters, e
    except Exception:
        return None, None


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def workload_config(cfg, shape, n_gpus, virtual=0):
    """The `config` object of BOTH arms (same keys and values, so the driver can pair the lines):
    what the workload is, never how an arm computes it."""
    cells = interior_cells(shape)
    return {"workload": cfg["workload"], "shape_zyx": list(shape), "iters": cfg["iters"],
            "parallelism": f"slab{n_gpus}" + (f" (virtual {virtual} slabs)" if virtual else ""),
            "l2": ("inputs larger than L2" if 8 * cells > L2_BYTES else "L2-resident (latency config)")}


def run_reference(args, cfg, shape, n_gpus):
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    from jacobi_inputs import u12
    field = u12(shape if shape[0] > 1 else shape[1:], 0x5C24)
    k_iter = args.ref_iters
    for _ in range(args.warmup):
        oracle_sample(shape, k_iter, field=field)
    vals, secs = [], []
    for _ in range(args.steps):
        v, dt, cores = oracle_sample(shape, k_iter, field=field)
        vals.append(v)
        secs.append(dt)
    value = interior_cells(shape) * k_iter * args.steps / sum(secs) / 1e9
    sample = f"{k_iter} of {cfg['iters']} iterations of the full {cfg['workload'].split(':')[0]} grid per step"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": n_gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(secs) / args.steps,
        "higher_is_better": True, "scaling": cfg["scaling"], "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (U12 seed 0x5C24)",
        "config": workload_config(cfg, shape, n_gpus),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "cpu_model": cpu_model(), "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "note": "no reference code exists (PAPER.md only); the reference arm is the CPU oracle (plain C, "
                "OpenMP over the outer axis) on this host's cores",
    }
    emit(line)
    return 0


_JSON_FD = None


def emit(line: dict) -> None:
    """The one JSON line on the real stdout (native libraries' prints were sent to stderr)."""
    os.write(_JSON_FD if _JSON_FD is not None else 1, (json.dumps(line) + "\n").encode())


def golden_digest(shape, iters):
    """The oracle digest of this workload (U12 seed 0x5C24, `iters` iterations), if committed."""
    want = list(shape if shape[0] > 1 else shape[1:])
    for fn in ("oracle_digests_full.json", "oracle_digests_latency.json", "oracle_digests.json"):
        try:
            with open(os.path.join(ROOT, "tests", "golden", fn)) as f:
                d = json.load(f)
        except OSError:
            continue
        for name, g in d.items():
            if g["shape"] == want and g["iters"] == iters and g.get("seed") == 0x5C24:
                return dict(g, name=name)
    return None


def assemble_field(h_out, shape, lo, hi, desc, world, rank, dist, torch):
    """The whole gathered field on rank 0: one process holds it in h_out already; with one rank
    per GPU every rank sends its owned outer planes (+ the global boundary plane it holds) to rank
    0 over torch.distributed (gloo, CPU tensors)."""
    import numpy as np
    nz, ny, nx = shape
    plane = nx * (ny if nz > 1 else 1)
    n_out = nz if nz > 1 else ny
    flat = h_out.numpy()
    if world == 1:
        return flat[: n_out * plane]
    start, chunk = desc["start"], desc["chunk"]
    a = start - 1 if start == 1 else start                     # first plane this rank owns / holds
    b = start + chunk + 1 if start + chunk == n_out - 1 else start + chunk
    mine = torch.from_numpy(np.ascontiguousarray(flat[(a - lo) * plane:(b - lo) * plane]))
    rng = torch.tensor([a, b], dtype=torch.int64)
    if rank != 0:
        dist.send(rng, 0)
        dist.send(mine, 0)
        return None
    full = np.empty(n_out * plane, dtype=np.float64)
    full[a * plane:b * plane] = mine.numpy()
    for r in range(1, world):
        dist.recv(rng, r)
        buf = torch.empty(int(rng[1] - rng[0]) * plane, dtype=torch.float64)
        dist.recv(buf, r)
        full[int(rng[0]) * plane:int(rng[1]) * plane] = buf.numpy()
    return full


def halo_latency(j, jb, modes, max_over_ranks, n=200):
    """Per-iteration time of no-compute runs (halo copies, flags and barriers only),
    (T(2n) - T(n)) / n to cancel the launch cost; µs.  Modes a handle does not support are
    reported as errors (e.g. the host-copy baselines in one-process-per-GPU mode)."""
    out = {}
    for name, mode in modes:
        try:
            j.set_mode(mode, jb.FLAG_NO_COMPUTE)
            j.run(n // 2)
            j.run(n)
            t1 = max_over_ranks(j.last_time_ms())
            j.run(2 * n)
            t2 = max_over_ranks(j.last_time_ms())
            out[name] = 1e3 * (t2 - t1) / n
        except jb.JacobiError as e:
            out[name] = {"error": str(e)}
    j.set_mode(jb.MODE_CPUFREE)
    return out


def traced_spans(j, jb, iters, n_trace, gather):
    """In-kernel %globaltimer spans of the boundary blocks (wait -> flag -> signal) over one
    CPU-Free run of the current workload; median over exchanges and slabs (skipping the first
    few exchanges of the launch), max over ranks via `gather`."""
    j.set_param("halo_trace", n_trace)
    try:
        j.run(iters)
        spans = []
        for i in range(j.local_slabs):
            spans.append(jb.halo_spans(j.halo_trace(i, min(n_trace, iters)), skip=min(8, iters // 4)))
    finally:
        j.set_param("halo_trace", 0)
    keys = ("wait_us", "put_us", "span_us", "period_us")
    res = {}
    for k in keys:
        v = [sp[k] for sp in spans if sp[k] is not None]
        res[k] = gather(max(v)) if v else None
    res["exchanges_per_slab"] = spans[0]["exchanges"] if spans else 0
    return res


def main():
    global _JSON_FD
    # stdout carries only the JSON line: NCCL and other native code print to fd 1 (e.g. "NCCL
    # version ..."), so fd 1 is pointed at stderr and the line is written to a saved copy.
    sys.stdout.flush()
    _JSON_FD = os.dup(1)
    os.dup2(2, 1)
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1,
                    help="GPUs: under torchrun one rank per GPU (WORLD_SIZE wins); without it one "
                         "process drives N GPUs (jacobi_create(ngpus=N), UVA peer stores)")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--iters", type=int, default=0, help="override iterations per step")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-iters", type=int, default=2, help="oracle iterations per reference step")
    ap.add_argument("--no-extras", action="store_true", help="skip e2e / cpu_baseline / baselines")
    ap.add_argument("--no-pipeline", action="store_true", help="skip the pipelined e2e (two fields)")
    ap.add_argument("--no-clocks", action="store_true", help="(diagnostic) no nvidia-smi sampling")
    ap.add_argument("--virtual", type=int, default=0, help="(measurement aid) P slabs on one GPU")
    ap.add_argument("--param", action="append", default=[], help="tuning knob name=value (jacobi_set_param)")
    ap.add_argument("--transport", default="ipc", choices=["ipc", "nvshmem"],
                    help="N>1: CUDA IPC peer stores (default) or the NVSHMEM variant (N3)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "ours" else args.warmup

    world, rank, local = dist_env()
    # N GPUs of the whole job: torchrun ranks, or --gpus in one process
    n_gpus = world if world > 1 else max(args.gpus, 1)
    single_multi = world == 1 and n_gpus > 1
    cfg = dict(CONFIGS[args.config])
    if args.iters:
        cfg["iters"] = args.iters
    shape = cfg["shape"] or (512 * n_gpus, 512, 512)  # C4 weak scaling: 512 z planes per GPU (R15)
    iters = cfg["iters"]

    if args.impl == "reference":
        return run_reference(args, cfg, shape, n_gpus)

    ndev = torch_device_count()
    if single_multi and ndev < n_gpus:
        # fail loudly (JACOBI_ENODEV): never measure fewer GPUs than asked for
        print(f"[bench] --gpus {n_gpus} needs {n_gpus} visible GPUs, found {ndev} (JACOBI_ENODEV)", file=sys.stderr)
        return 2
    if world > 1 and ndev < 1:
        print("[bench] no GPU visible to this rank (JACOBI_ENODEV)", file=sys.stderr)
        return 2
    local = local % max(ndev, 1)  # (more ranks than GPUs only in functional tests: time-sliced)

    import numpy as np
    import torch
    import paper_conf_sc_baydamirlibu24_b200 as jb

    torch.cuda.set_device(local)
    if world > 1 and args.transport == "nvshmem":
        import torch.distributed as dist
        dist.init_process_group("gloo")
        j = jb.create_nvshmem(shape, device=local)  # symmetric heap owns the slabs
        args.no_extras = True  # CPU-controlled baselines / e2e use the IPC build
    elif world > 1:
        jb.use_torch_allocator()  # PyTorch owns the device memory of the slabs (north star)
        import torch.distributed as dist
        dist.init_process_group("gloo")
        j = jb.Jacobi(shape, dist=(rank, world), device=local)
        jb.exchange_peers(j, nccl=False)
        try:  # NCCL comm of the CPU-controlled baseline (needs one GPU per rank)
            uid = jb.broadcast_blob(jb.jacobi_nccl_unique_id() if rank == 0 else None)
            jb.jacobi_nccl_init(j.h, uid)
        except jb.JacobiError as e:
            print(f"[bench] NCCL baseline unavailable: {e}", file=sys.stderr)
    else:
        jb.use_torch_allocator()
        dist = None
        j = jb.Jacobi(shape, virtual=args.virtual) if args.virtual else jb.Jacobi(shape, ngpus=n_gpus)
    torch.cuda.set_device(local)
    for kv in args.param:
        k, v = kv.split("=")
        j.set_param(k, int(v))

    def barrier():
        if dist is not None:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    def sync_all():
        for d in range(ndev if single_multi else 0):
            torch.cuda.synchronize(d)
        torch.cuda.synchronize(local)

    cells = interior_cells(shape)
    desc = j.describe(0)  # slab 0 owns the largest chunk (the first r slabs get one more plane)
    per_plane = cells // (shape[0] - 2 if shape[0] > 1 else shape[1] - 2)
    local_cells = per_plane * desc["chunk"] if n_gpus > 1 else cells  # cells of the busiest GPU

    # ---- warm-up + timed region (device time per launch from CUDA events on the launch stream)
    for _ in range(args.warmup):
        j.run(iters)
    barrier()
    sync_all()
    clocks = ClockSampler(local) if rank == 0 and not args.no_clocks else None
    if clocks:
        clocks.start()
    t_wall0 = time.perf_counter()
    step_ms = []
    launches = 0
    for _ in range(args.steps):
        j.run(iters)
        step_ms.append(j.last_time_ms())  # max over this process's GPUs
        launches += j.get_param("last_launches")
    sync_all()
    barrier()
    t_wall = time.perf_counter() - t_wall0
    clk = clocks.stop() if clocks else None
    dev_ms_local = sum(step_ms)
    dev_ms = max_over_ranks(dev_ms_local)
    value = cells * iters * args.steps / (dev_ms / 1e3) / 1e9
    launches = int(sum_over_ranks(launches))

    # ---- roofline of the dominant kernel.  Per cell-update it moves 16 B (read once + write
    #      once) when it runs one iteration per pass over HBM, 16/K B when the
    #      temporally blocked kernel runs K iterations per pass.  Per GPU: the
    #      busiest GPU's cells over its launch time.
    peak, peak_kind = measured_hbm()
    launch_ms = dev_ms / args.steps
    tb_iters = jb.jacobi_get_param(j.h, "last_tblock")
    tb_k = max(jb.jacobi_get_param(j.h, "last_tb_k"), 1)
    resident = bool(jb.jacobi_get_param(j.h, "last_resident"))
    cluster_nc = jb.jacobi_get_param(j.h, "last_cluster")
    alg_bytes = round(local_cells * (16 * (iters - tb_iters) + 16 / tb_k * tb_iters))
    achieved = alg_bytes / (launch_ms / 1e3) / 1e9
    dimk = 2 if shape[0] == 1 else 3
    if tb_iters:
        kname = f"jb_tblock<{dimk},{tb_k},*> (persistent CPU-Free kernel, {tb_k} iterations per HBM pass)"
        kkind = "tblock"
    elif cluster_nc:
        kname = f"jb_cluster2d (one {cluster_nc}-CTA thread-block cluster, grid on chip, DSMEM halos, cluster barrier)"
        kkind = "cluster"
    elif resident:
        kname = f"jb_resident<{dimk},*> (persistent CPU-Free kernel, on-chip resident)"
        kkind = "resident"
    else:
        kname = f"jb_sweep<{dimk},false,true,false> (persistent CPU-Free kernel, streaming)"
        kkind = "streaming"
    l2_resident = 8 * cells <= L2_BYTES
    us_per_iter = 1e3 * launch_ms / iters
    if l2_resident:
        # C1 / C5: the field lives in L2 (or on chip), so HBM is not the bound: latency per
        # iteration (grid barrier + flag round trip) is the figure of merit
        roofline = {"bound": "latency", "achieved": us_per_iter, "peak": None, "unit": "us/iteration",
                    "frac": None, "traffic": None, "kernel": kname,
                    "note": "L2-resident latency config: microseconds per iteration, not an HBM fraction"}
    else:
        traffic, _ = ncu_traffic(args.config + ("_tblock" if tb_iters else ""), iters)
        roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                    "frac": achieved / peak, "traffic": traffic, "peak_kind": peak_kind,
                    "kernel": kname, "alg_bytes_per_launch": alg_bytes,
                    "alg_bytes_per_cell_update": alg_bytes / (local_cells * iters),
                    "per_gpu": n_gpus > 1}
        if tb_iters:
            # K iterations per HBM pass move 16/K B per update, so HBM is no longer the only ceiling:
            # (a) the bandwidth a one-iteration-per-pass kernel would need for the same throughput
            #     (16 B per update; > the HBM peak means the time blocking beat the HBM roofline);
            # (b) the fp64 pipe: 3 DADD + 1 DMUL (2D) / 5 + 1 (3D) per update, no FMA (oracle order),
            #     64 fp64 lanes per SM per clock (B200 vector fp64 ~37 TFLOP/s; ncu's
            #     sm__pipe_fp64_cycles_active agrees: DESIGN.md §5.8), 148 SMs at the max SM clock.
            sm_mhz = (clk or {}).get("sm_max_mhz") or 1965.0
            fp64_peak = 64 * 148 * sm_mhz * 1e6
            ops = 4 if dimk == 2 else 6
            roofline["equivalent_gbs_at_16B"] = 16 * local_cells * iters / (launch_ms / 1e3) / 1e9
            roofline["equivalent_frac_at_16B"] = roofline["equivalent_gbs_at_16B"] / peak
            roofline["fp64_pipe"] = {"achieved_ops": ops * local_cells * iters / (launch_ms / 1e3),
                                     "peak_ops": fp64_peak,
                                     "frac": ops * local_cells * iters / (launch_ms / 1e3) / fp64_peak,
                                     "ops_per_update": ops,
                                     "peak_basis": "64 fp64 lanes/SM/clk x 148 SMs x max SM clock (DESIGN.md 5.8)"}

    transport = ("none" if n_gpus == 1 else
                 "nvshmem" if (world > 1 and args.transport == "nvshmem") else
                 "cuda-ipc peer stores (one process per GPU)" if world > 1 else
                 "UVA peer stores (one process, cudaDeviceEnablePeerAccess)")
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": n_gpus, "steps": args.steps,
        "transport": transport,
        "warmup": args.warmup, "ms_per_step": dev_ms / args.steps, "higher_is_better": True,
        "scaling": cfg["scaling"], "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (U12 seed 0x5C24, initialised on the device)",
        "config": workload_config(cfg, shape, n_gpus, args.virtual),
        "kernel_config": {"kernel": kkind,
                          "tile": {k: desc[k] for k in ("tile_x", "tile_y", "stages", "ctas", "n_top", "n_bot",
                                                        "k_planes")},
                          **({"time_block": {"K": tb_k, "iters_time_blocked": tb_iters,
                                             "note": "tile above is the per-iteration plan; the time-blocked "
                                                     "kernel's strips/tiles are in DESIGN.md 5.8-5.9"}}
                             if tb_iters else {})},
        "gpu_launches": launches,
        "wall_ms_per_step": 1e3 * t_wall / args.steps,
        "ms_per_iter": dev_ms / args.steps / iters,
        "us_per_iter": us_per_iter,
        "roofline": roofline,
        "clocks": clk,
    }

    if not args.no_extras:
        # ---- this box's own copy bandwidth (same method as MEASURED_PEAKS.json: torch copy_ of
        #      1 Gi bf16 elements, read + write bytes, best of 10), for context beside `roofline`
        try:
            a = torch.empty(1 << 30, dtype=torch.bfloat16, device=f"cuda:{local}")
            b = torch.empty_like(a)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            best = None
            for _ in range(10):
                e0.record()
                b.copy_(a)
                e1.record()
                e1.synchronize()
                ms = e0.elapsed_time(e1)
                best = ms if best is None else min(best, ms)
            box_copy = 2 * a.numel() * a.element_size() / (best / 1e3) / 1e9
            if roofline["bound"] == "hbm":
                line["roofline"]["box_copy_gbs"] = box_copy
                line["roofline"]["frac_of_box_copy"] = line["roofline"]["achieved"] / box_copy
            del a, b
            torch.cuda.empty_cache()
        except Exception as e:  # never fail the bench line for a context number
            print(f"[bench] box copy measurement failed: {e}", file=sys.stderr)

        # ---- the per-iteration CPU-Free kernel (one iteration per HBM pass, the paper's Listing
        #      4.1 structure) on the same workload, for comparison with the time-blocked one
        if tb_iters:
            j.set_param("tblock", 0)
            j.run(iters)
            ms1 = []
            for _ in range(args.steps):
                j.run(iters)
                ms1.append(j.last_time_ms())
            j.set_param("tblock", -1)
            ms1 = max_over_ranks(sum(ms1))
            v1 = cells * iters * args.steps / (ms1 / 1e3) / 1e9
            a1 = 16 * local_cells * iters / (ms1 / args.steps / 1e3) / 1e9
            line["per_iteration_kernel"] = {"value": v1, "unit": UNIT, "kernel": "jb_sweep (streaming)",
                                            "achieved_gbs": a1, "frac": a1 / peak,
                                            "alg_bytes_per_cell_update": 16}

        # ---- CPU-controlled baselines (per-iteration launch + copy/NCCL + host sync), short run
        base = {}
        b_iters = min(iters, 200)
        # (NCCL needs one GPU per rank: not with virtual slabs sharing one GPU)
        bmodes = [("memcpy", jb.MODE_BASELINE_MEMCPY)] + ([] if args.virtual > 1 else [("nccl", jb.MODE_BASELINE_NCCL)])
        if single_multi:
            bmodes += [("overlap", jb.MODE_BASELINE_OVERLAP), ("p2p", jb.MODE_BASELINE_P2P),
                       ("graph", jb.MODE_BASELINE_GRAPH)]
        for name, mode in bmodes:
            if world > 1 and name == "memcpy":
                continue  # host peer copies need one process (dist mode: NCCL)
            try:
                j.set_mode(mode)
                j.run(b_iters)  # warm
                j.run(b_iters)
                ms = max_over_ranks(j.last_time_ms())
                base[name] = {"value": cells * b_iters / (ms / 1e3) / 1e9, "unit": UNIT,
                              "ms_per_iter": ms / b_iters, "iters": b_iters}
            except jb.JacobiError as e:
                base[name] = {"error": str(e)}
        j.set_mode(jb.MODE_CPUFREE)
        line["cpu_controlled"] = base

        # ---- per-iteration halo latency (no-compute runs) and NVLink evidence at N > 1
        if n_gpus > 1 or args.virtual > 1:
            hmodes = [("cpufree", jb.MODE_CPUFREE)] + ([] if args.virtual > 1 else [("baseline_nccl", jb.MODE_BASELINE_NCCL)])
            if world == 1:
                hmodes += [("baseline_memcpy", jb.MODE_BASELINE_MEMCPY), ("baseline_graph", jb.MODE_BASELINE_GRAPH)]
            halo = halo_latency(j, jb, hmodes, max_over_ranks)
            nz, ny, nx = shape
            plane_bytes = 8 * nx * (ny if nz > 1 else 1)  # one halo message = one outer plane
            sides = 2 if n_gpus > 2 or args.virtual > 2 else 1  # interior GPUs send to both neighbours
            msg = {"halo_bytes_per_iter_per_gpu_out": sides * plane_bytes,
                   "halo_bytes_per_iter_per_gpu_in": sides * plane_bytes,
                   "message_bytes": plane_bytes, "nvlink_peak_gbs_per_direction": 900.0}
            if isinstance(halo.get("cpufree"), float) and halo["cpufree"] > 0:
                gbs = sides * plane_bytes / (halo["cpufree"] * 1e-6) / 1e9
                msg["achieved_gbs_per_direction_nocompute"] = gbs
                msg["frac_of_nvlink"] = gbs / 900.0
            # every CPU-Free kernel delivers one outer plane per side and iteration (the
            # time-blocked one as its K edge-zone phases: level-m planes into the neighbour's
            # slots, the last into its halo), so the halo rate of the timed compute run is:
            gbs = sides * plane_bytes / (1e-3 * launch_ms / iters) / 1e9
            msg["halo_gbs_during_compute_run"] = gbs
            msg["halo_frac_of_nvlink_during_compute_run"] = gbs / 900.0
            line["halo_us"] = halo
            line["halo_traffic"] = msg
            if args.virtual > 1:
                line["halo_traffic"]["note"] = "virtual slabs share one GPU: no NVLink traffic"
            # in-kernel spans of the boundary blocks: the compute run of the timed kernel and a
            # no-compute run (flag round trip + barrier only)
            try:
                n_tr = min(iters, 1024)
                line["halo_spans_compute"] = traced_spans(j, jb, iters, n_tr, max_over_ranks)
                j.set_mode(jb.MODE_CPUFREE, jb.FLAG_NO_COMPUTE)
                line["halo_spans_nocompute"] = traced_spans(j, jb, 400, 400, max_over_ranks)
                j.set_mode(jb.MODE_CPUFREE)
            except jb.JacobiError as e:
                line["halo_spans_compute"] = {"error": str(e)}
                j.set_mode(jb.MODE_CPUFREE)
        else:
            line["halo_us"] = None  # one slab: no halo; see bench_latency.py (virtual slabs)
            # Context at N = 1: the same grid split into 2 VIRTUAL slabs on this GPU (thread-block
            # groups running the complete flag / halo protocol; no NVLink), no-compute per-iteration
            # time of the CPU-Free kernel vs the CPU-controlled baselines.
            try:
                with jb.Jacobi(shape, virtual=2) as jv:
                    line["halo_us_virtual2"] = dict(
                        halo_latency(jv, jb, [("cpufree", jb.MODE_CPUFREE),
                                              ("baseline_memcpy", jb.MODE_BASELINE_MEMCPY),
                                              ("baseline_graph", jb.MODE_BASELINE_GRAPH)], lambda x: x),
                        note="2 virtual slabs of this grid on one GPU (no NVLink); us per no-compute iteration")
            except (jb.JacobiError, ValueError) as e:
                line["halo_us_virtual2"] = {"error": str(e)}

        # ---- e2e through the C ABI with pinned host buffers (scatter + run + gather per step)
        from jacobi_inputs import u12_flat
        nz, ny, nx = shape
        plane = nx * (ny if nz > 1 else 1)
        n_out = nz if nz > 1 else ny
        start, chunk = desc["start"], desc["chunk"]
        if world > 1:
            lo, hi = start - 1, start + chunk + 1  # this rank's slab + halos
        else:
            lo, hi = 0, n_out
        nbytes = (hi - lo) * plane * 8
        h_in = torch.empty((hi - lo) * plane, dtype=torch.float64, pin_memory=True)
        h_out = torch.empty((hi - lo) * plane, dtype=torch.float64, pin_memory=True)
        h_in.numpy()[:] = u12_flat(lo * plane, (hi - lo) * plane, 0x5C24)
        base_in = h_in.data_ptr() - lo * plane * 8
        base_out = h_out.data_ptr() - lo * plane * 8
        if world > 1:
            d2h = (chunk + (1 if start == 1 else 0) + (1 if start + chunk == n_out - 1 else 0)) * plane * 8
        else:
            d2h = n_out * plane * 8
        jb.jacobi_scatter_ptr(j.h, base_in)
        j.run(iters)
        jb.jacobi_gather_ptr(j.h, base_out)
        barrier()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            jb.jacobi_scatter_ptr(j.h, base_in)
            j.run(iters)
            jb.jacobi_gather_ptr(j.h, base_out)
        barrier()
        e2e_s = max_over_ranks(time.perf_counter() - t0)
        h2d_total = sum_over_ranks(float(nbytes))
        d2h_total = sum_over_ranks(float(d2h))
        line["e2e"] = {"value": cells * iters * args.steps / e2e_s / 1e9, "unit": UNIT,
                       "h2d_bytes_per_step": int(h2d_total), "d2h_bytes_per_step": int(d2h_total),
                       "ms_per_step": 1e3 * e2e_s / args.steps,
                       "path": "jacobi_scatter (pinned H2D) + jacobi_run + jacobi_gather (pinned D2H)"}

        # ---- e2e, pipelined (one process): two fields on the device; while one step runs, a second
        #      host thread gathers the previous step's result and scatters the next step's input on
        #      the other field, through the same public calls (H2D / D2H overlap the compute; every
        #      step still copies its whole input in and its whole result out inside the timed region)
        if world == 1 and args.steps >= 2 and not args.no_pipeline:
            import threading
            j2 = jb.Jacobi(shape, virtual=args.virtual) if args.virtual else jb.Jacobi(shape, ngpus=n_gpus)
            for kv in args.param:
                k, v = kv.split("=")
                j2.set_param(k, int(v))
            hs = [j, j2]
            h_out2 = torch.empty_like(h_out, pin_memory=True)
            outs = [h_out.data_ptr() - lo * plane * 8, h_out2.data_ptr() - lo * plane * 8]
            j2.run(iters)  # warm the second handle's plan
            err = []

            def copies(i):
                try:
                    if i >= 1:
                        jb.jacobi_gather_ptr(hs[(i - 1) % 2].h, outs[(i - 1) % 2])
                    if i + 1 < args.steps:
                        jb.jacobi_scatter_ptr(hs[(i + 1) % 2].h, base_in)
                except Exception as e:  # noqa: BLE001
                    err.append(e)

            t0 = time.perf_counter()
            jb.jacobi_scatter_ptr(hs[0].h, base_in)
            for i in range(args.steps):
                th = threading.Thread(target=copies, args=(i,))
                th.start()
                hs[i % 2].run(iters)
                th.join()
            jb.jacobi_gather_ptr(hs[(args.steps - 1) % 2].h, outs[(args.steps - 1) % 2])
            e2p_s = time.perf_counter() - t0
            if err:
                raise err[0]
            same = bool(np.array_equal(h_out.numpy().view(np.uint64), h_out2.numpy().view(np.uint64)))
            line["e2e_pipelined"] = {"value": cells * iters * args.steps / e2p_s / 1e9, "unit": UNIT,
                                     "h2d_bytes_per_step": int(nbytes), "d2h_bytes_per_step": int(d2h),
                                     "ms_per_step": 1e3 * e2p_s / args.steps, "fields": 2,
                                     "results_identical": same,
                                     "path": "two handles: jacobi_run of step i || (jacobi_gather of step i-1 + "
                                             "jacobi_scatter of step i+1) on a second host thread"}
            j2.close()
            del h_out2

        # ---- parity of the measured configuration: the e2e step above scattered the U12 field and
        #      ran exactly `iters` iterations through the C ABI on these N GPUs, so the gathered
        #      field is compared (SHA-256 of the whole field) with the digest of the CPU oracle's
        #      own run of that workload, where tests/golden holds one (C1, C2, C3 at their
        #      lengths; written by tests/golden/make_golden.py from oracle/ only)
        gold = golden_digest(shape, iters)
        if gold is not None:
            full = assemble_field(h_out, shape, lo, hi, desc, world, rank, dist, torch)
            if rank == 0:
                import hashlib
                got = hashlib.sha256(np.ascontiguousarray(full).tobytes()).hexdigest()
                line["parity"] = {"match": got == gold["sha256"], "sha256": got, "oracle_sha256": gold["sha256"],
                                  "what": f"whole {shape} field after {iters} iterations on {n_gpus} GPU(s) "
                                          f"(e2e step) vs the oracle digest {gold['name']}"}

        # ---- CPU oracle on this host's cores (rank 0, N = 1 only), bounded sample
        if rank == 0 and n_gpus == 1:
            field = h_in.numpy().reshape(shape if nz > 1 else shape[1:])
            v1, dt1, cores = oracle_sample(shape, 1, field=field)
            k = int(max(1, min(50, 10.0 / max(dt1, 1e-3))))
            v, dt, cores = oracle_sample(shape, k, field=field)
            line["cpu_baseline"] = {"value": v, "unit": UNIT, "cores": cores, "cpu_model": cpu_model(),
                                    "kind": "oracle",
                                    "sample": f"{k} of {iters} iterations on the full grid "
                                              f"({dt:.1f} s, OpenMP over the outer axis)"}
    if rank == 0:
        emit(line)
    j.close()
    if args.transport == "nvshmem" and world > 1:
        jb.nvshmem_finalize()
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
