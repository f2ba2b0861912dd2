"""Benchmark: fused Q-criterion on a 1024^3 fp32 rectilinear mesh per GPU.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Workload (BASELINE.json metric / configs[3]): synthetic
Rayleigh-Taylor-like velocity (synth/), non-uniform x/y/z coordinates, the
Q-criterion program of Fig. 3C (completed per DESIGN.md
G1-G3), fused strategy.  N > 1: weak scaling, every rank owns a 1024^3 z-slab
of a 1024 x 1024 x (1024 N) mesh, one ghost plane per side exchanged with
NCCL inside dfg_execute.  One step = one dfg_execute (halo + fused kernel)
with inputs resident in HBM; value = cells/s of the whole job.

Prints ONE JSON line on rank 0.  See DESIGN.md section 7 for every key.
"""

from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Q-criterion cells/sec & HBM GB/s (fused vs staged vs roundtrip), 1/2/4/8 B200"
N1 = 1024                       # cells per axis per GPU
ALGO_BYTES_PER_CELL = 16        # fused Q, fp32: u, v, w read once + q written once


def _peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._ready = threading.Event()   # first sample taken (NVML initialised)
        self._t = None

    # NVML clocks-event reason bits (nvml.h): sw power cap, hw slowdown,
    # sw thermal slowdown, hw thermal slowdown
    BITS = ((0x8, 3), (0x40, 4), (0x20, 5), (0x4, 6))

    def _run(self):
        try:  # NVML: a query takes microseconds, so ~100 samples per second
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            get_reasons = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                pynvml.nvmlDeviceGetCurrentClocksThrottleReasons
            while not self._stop.is_set():
                sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                pw = pynvml.nvmlDeviceGetPowerUsage(h) / 1000.0
                bits = get_reasons(h)
                row = [str(sm), str(mx), f"{pw:.1f}", "", "", "", ""]
                for bit, col in self.BITS:
                    row[col] = "Active" if bits & bit else "Not Active"
                self.rows.append(row)
                self._ready.set()
                self._stop.wait(0.002)
            self.source = "nvml"
            return
        except Exception:
            pass
        self.source = "nvidia-smi"
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.rows.append([c.strip() for c in out.split(",")])
                    self._ready.set()
            except Exception:
                pass
            self._stop.wait(0.05)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        # the timed region starts only once sampling runs (NVML init can take
        # longer than a short timed region)
        self._ready.wait(timeout=10.0)
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 3 + i and r[3 + i] == "Active"})
        pw = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "power_w": float(np.median(pw)) if pw else None,
                "reasons": reasons, "samples": len(self.rows), "source": getattr(self, "source", None)}


def host_cpu():
    """lscpu model / sockets / cores of the host the CPU baselines run on
    (report the oracle's hardware with its number)."""
    info = {"nproc": os.cpu_count()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            k, v = k.strip(), v.strip()
            if k in ("Model name", "Socket(s)", "Core(s) per socket", "Thread(s) per core", "CPU(s)"):
                info[k.lower().replace("(s)", "s").replace(" ", "_")] = v
    except Exception as e:  # no lscpu on this host
        info["lscpu"] = repr(e)[:100]
    return info


# ------------------------------------------------------------------ oracle
def _oracle_sample(nx_rows: int, planes: int, k0: int = 100, j0: int = 200, fields=None):
    """Inputs for an oracle sample: a 1024 x nx_rows x planes block of the
    bench mesh (plus its one-cell halo): the window of the GPU's own input
    arrays when given (the same inputs on both sides), else generated on the
    CPU (the CPU and CUDA generators agree except for rare fp32 rounding
    flips: their fp64 sin / log differ in the last bit)."""
    import torch

    import synth
    x, y, z = synth.rt_coords(N1, N1, N1, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    k1 = k0 + planes
    j1 = j0 + nx_rows
    win = (k0 - 1, k1 + 1, j0 - 1, j1 + 1, 0, N1)
    if fields is not None:
        f = {c: fields[c][win[0]:win[1], win[2]:win[3], :].cpu().numpy() for c in "uvw"}
    else:
        f = {c: synth.rt_velocity(c, x64, y64, z64, win, torch.float32).numpy() for c in "uvw"}
    return x, y, z, f, win


def _oracle_time(x, y, z, f, win):
    from oracle import evaluate as oev
    from oracle.lang import QCRIT, build_dag
    dag = build_dag(QCRIT, ("u", "v", "w"), "f32")
    t0 = time.perf_counter()
    res, valid = oev.evaluate(dag, f, oev.MeshWindow(x, y, z, i0=win[4], j0=win[2], k0=win[0]))
    dt = time.perf_counter() - t0
    cells = int(valid[1:-1, 1:-1, :].sum())
    return cells, dt, res[1:-1, 1:-1, :]


def _oracle_mt_worker(i, nworkers, barrier, target_s):
    """One process of the multi-core oracle timing: its own block of the
    bench mesh (64 rows x 4 planes, distinct per worker), evaluated by the
    unchanged oracle repeatedly for about target_s once every worker is ready."""
    planes, rows = 4, 64
    k0 = 8 + (i * planes) % (N1 - 16)
    j0 = 64 + 64 * ((i * planes) // (N1 - 16)) % (N1 - 128)
    x, y, z, f, win = _oracle_sample(rows, planes, k0, j0)
    _oracle_time(x, y, z, f, win)                              # warm (page-in, allocator)
    barrier.wait()
    t0 = time.time()
    cells = 0
    while True:
        c, _, _ = _oracle_time(x, y, z, f, win)
        cells += c
        if time.time() - t0 >= target_s:
            break
    return cells, t0, time.time()


def cpu_baseline_mt(target_s: float = 8.0):
    """oracle_mt: the same oracle in one single-threaded process
    per host core (capped at 64 for memory), each on its own block; throughput =
    all cells / (last end - first start).  The arithmetic is the oracle's."""
    import multiprocessing as mp
    n = max(1, min(64, os.cpu_count() or 1))
    for k in ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS"):
        os.environ[k] = "1"
    ctx = mp.get_context("spawn")
    with ctx.Manager() as mgr:
        barrier = mgr.Barrier(n)
        with ctx.Pool(n) as pool:
            res = pool.starmap(_oracle_mt_worker, [(i, n, barrier, target_s) for i in range(n)])
    cells = sum(r[0] for r in res)
    wall = max(r[2] for r in res) - min(r[1] for r in res)
    return {"value": cells / wall, "unit": "cells/s", "cores": n, "kind": "oracle",
            "sample": f"{n} processes x repeated Q-criterion on 1024 x 64 x 4 blocks of the 1024^3 RT-like fp32 "
                      f"workload, numpy oracle, {wall:.1f} s wall"}


def cpu_baseline_leg(target_s: float = 12.0, gpu_out=None, gpu_fields=None):
    """The oracle as it stands (numpy, one thread for element-wise ops) on a
    bounded sample of the bench workload.  With gpu_out / gpu_fields (the fused
    kernel's 1024^3 result of the timed steps and its inputs), the sample runs
    on the GPU's own inputs and doubles as a full-size parity check: the GPU
    cells of the block must equal the oracle's bit for bit."""
    x, y, z, f, win = _oracle_sample(512, 4)
    cells, dt, _ = _oracle_time(x, y, z, f, win)                 # calibration run
    planes = int(max(1, min(128, round(4 * target_s / max(dt, 1e-3)))))
    x, y, z, f, win = _oracle_sample(512, planes, fields=gpu_fields)
    cells, dt, res = _oracle_time(x, y, z, f, win)
    line = {"value": cells / dt, "unit": "cells/s", "cores": 1, "kind": "oracle", "host": host_cpu(),
            "sample": f"Q-criterion on a 1024 x 512 x {planes} block (+1-cell halo) of the 1024^3 RT-like "
                      f"fp32 workload, numpy oracle, {dt:.1f} s"}
    if gpu_out is not None:
        k0, j0 = win[0] + 1, win[2] + 1
        got = gpu_out[k0:k0 + res.shape[0], j0:j0 + res.shape[1], :].cpu().numpy()
        line["gpu_parity"] = {"cells_compared": int(res.size),
                              "mismatches": int(np.count_nonzero(got.view(np.uint32) != res.view(np.uint32))),
                              "block": f"planes {k0}..{k0 + res.shape[0] - 1}, rows {j0}..{j0 + res.shape[1] - 1}"}
    return line


def run_reference(args):
    """--impl reference: the oracle is this tier's reference arm (CPU only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    K, W = args.steps, args.warmup
    budget = 150.0
    x, y, z, f, win = _oracle_sample(16, 4)
    _, dt, _ = _oracle_time(x, y, z, f, win)
    per_step = budget / (K + W)
    scale = 16 * per_step / max(dt, 1e-3)          # in rows of 1024 x 1 x 4 cells
    rows = int(max(1, min(800, round(scale))))
    planes = int(4 * max(1, min(100, round(scale / rows))))
    x, y, z, f, win = _oracle_sample(rows, planes)
    for _ in range(W):
        _oracle_time(x, y, z, f, win)
    tot_cells, tot_t = 0, 0.0
    for _ in range(K):
        c, dt, _ = _oracle_time(x, y, z, f, win)
        tot_cells += c
        tot_t += dt
    v = tot_cells / tot_t
    sample = (f"each step: Q-criterion on a 1024 x {rows} x {planes} block (+1-cell halo) of the RT-like "
              f"workload, numpy oracle")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "cells/s", "n_gpus": args.gpus,
            "steps": K, "warmup": W, "ms_per_step": 1e3 * tot_t / K, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": "fused Q-criterion 1024^3 fp32 per GPU (oracle: bounded CPU sample)",
                       "expression": "qcrit"},
            "cpu_baseline": {"value": v, "unit": "cells/s", "cores": 1, "kind": "oracle", "sample": sample,
                             "host": host_cpu()},
            "e2e": {"value": v, "unit": "cells/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def slab_boundary_parity(dist, torch, rank, world, fields, out, x, y, z, n, nzl, g, target_s=10.0):
    """N > 1: the oracle against the GPU on rank 0's slab where the halo
    matters -- a block of full rows ending at the slab's LAST owned plane,
    whose z+1 neighbours live on rank 1 (ghost data lets the
    gradient compute the proper values on the boundaries).  Rank 1 sends its
    first owned plane of u, v, w (the window's rows) to rank 0; rank 0 runs
    the unchanged oracle on its own planes + that plane and compares the
    last planes of its output bit for bit.  Every other rank only joins the
    exchange.  Returns the rank-0 cpu_baseline line (or None elsewhere)."""
    j0 = min(200, n // 4)
    rows = min(512, n - j0 - 1)
    win_rows = slice(j0 - 1, j0 + rows + 1)
    if rank == 1:
        t = torch.stack([fields[c][g, win_rows, :] for c in "uvw"]).contiguous()
        dist.send(t, dst=0)
        return None
    if rank != 0:
        return None
    recv = torch.empty((3, rows + 2, n), dtype=torch.float32, device="cuda")
    dist.recv(recv, src=1)
    from oracle import evaluate as oev
    from oracle.lang import QCRIT, build_dag
    dag = build_dag(QCRIT, ("u", "v", "w"), "f32")

    def sample(planes):
        k0 = nzl - planes                            # global = local on rank 0 (z_offset 0)
        f = {}
        for i, c in enumerate("uvw"):
            own = fields[c][g + k0 - 1:g + nzl, win_rows, :].cpu().numpy()
            f[c] = np.concatenate([own, recv[i:i + 1].cpu().numpy()], axis=0)
        t0 = time.perf_counter()
        res, valid = oev.evaluate(dag, f, oev.MeshWindow(x, y, z, i0=0, j0=j0 - 1, k0=k0 - 1))
        return k0, res[1:-1, 1:-1, :], int(valid[1:-1, 1:-1, :].sum()), time.perf_counter() - t0

    _, _, _, dt = sample(2)                          # calibration
    planes = int(max(2, min(64, nzl - 1, round(2 * target_s / max(dt, 1e-3)))))
    k0, res, cells, dt = sample(planes)
    got = out[k0:nzl, j0:j0 + rows, :].cpu().numpy()
    bad = int(np.count_nonzero(got.view(np.uint32) != res.view(np.uint32)))
    return {"value": cells / dt, "unit": "cells/s", "cores": 1, "kind": "oracle", "host": host_cpu(),
            "sample": f"Q-criterion on a {n} x {rows} x {planes} block of rank 0's slab ending at its last owned "
                      f"plane (z+1 neighbours from rank 1), numpy oracle, {dt:.1f} s",
            "slab_boundary_parity": {"cells_compared": int(res.size), "mismatches": bad,
                                     "block": f"planes {k0}..{nzl - 1} (slab boundary at {nzl - 1}|{nzl}), "
                                              f"rows {j0}..{j0 + rows - 1}"}}


def _self_launch(args):
    """--gpus N > 1 outside torchrun: run this script under
    torch.distributed.run with N ranks (one per GPU, rendezvous on
    127.0.0.1), the launch the driver uses; fail loudly when the node has
    fewer GPUs (DFG_BENCH_ONE_GPU=1: every rank on cuda:0, functional test)."""
    import socket

    import torch
    have = torch.cuda.device_count()
    if os.environ.get("DFG_BENCH_ONE_GPU") != "1" and have < args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} needs {args.gpus} CUDA devices, this node has {have} "
                         "(DFG_BENCH_ONE_GPU=1 runs every rank on cuda:0 as a functional test)\n")
        return 2
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


# ---------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--size", type=int, default=N1, help="cells per axis per GPU (default 1024)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-strategies", action="store_true")
    ap.add_argument("--no-cpu-mt", action="store_true", help="skip the multi-process oracle timing")
    ap.add_argument("--halo", default="auto", choices=["auto", "peer", "nccl"],
                    help="N > 1 z-slab halo: peer memory read in place by the kernel, NCCL send/recv, or auto "
                         "(default): peer when every rank's isolated probe of the in-place TMA read passes, else NCCL")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: size^3 cells per GPU (mesh size x size x size*N); strong: one size^3 mesh "
                         "split into N z-slabs (config 4 of BASELINE.json runs both)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return _self_launch(args)
    if int(os.environ.get("WORLD_SIZE", "1")) != args.gpus:
        sys.stderr.write(f"bench.py: WORLD_SIZE={os.environ.get('WORLD_SIZE')} but --gpus {args.gpus}\n")
        return 2
    global ORACLE_CHECKS
    ORACLE_CHECKS = not args.no_cpu_baseline

    import torch
    import torch.distributed as dist

    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    import synth
    QCRIT = dfg.paper_program("qcrit")  # the paper's program text, from the library

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # Test hook, not a measurement: DFG_BENCH_ONE_GPU=1 puts every rank on cuda:0
    # with its own NCCL_HOSTID (NCCL then uses its socket transport), so the
    # N > 1 path runs end to end on a one-GPU box; its timings mean nothing.
    one_gpu = world > 1 and os.environ.get("DFG_BENCH_ONE_GPU") == "1"
    if one_gpu:   # torch's own NCCL process group needs it too
        os.environ.update({"NCCL_HOSTID": f"dfg-bench-{rank}", "NCCL_SOCKET_IFNAME": "lo", "NCCL_IB_DISABLE": "1",
                           "NCCL_P2P_DISABLE": "1", "NCCL_SHM_DISABLE": "1"})
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    n = args.size
    NZ = n * world if args.scaling == "weak" else n
    K, W = args.steps, args.warmup
    assert W >= 3, "at least 3 warm-up steps"

    # mesh + inputs (slab of rank r with one ghost plane per side when N > 1)
    x, y, z = synth.rt_coords(n, n, NZ, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    k0, nzl = dfg.dfg_partition(NZ, world, rank)
    g = 1 if world > 1 else 0
    fields = {}
    for c in "uvw":
        buf = torch.zeros((nzl + 2 * g, n, n), dtype=torch.float32, device="cuda")
        buf[g:g + nzl] = synth.rt_velocity(
            c, x64, y64, z64, (k0, k0 + nzl, 0, n, 0, n), torch.float32, "cuda")
        fields[c] = buf
    mesh = dfg.Mesh(x, y, z, nz_local=nzl, z_offset=k0, ghost=g)
    for c, b in fields.items():
        mesh.bind(c, b)
    halo = None
    probe = None
    if world > 1:
        halo = "nccl"
        if args.halo in ("peer", "auto"):
            # the kernel reads the neighbours' boundary planes in place (CUDA IPC
            # mappings over NVLink); every rank must link or none does.  auto:
            # first an isolated probe (a child process per rank TMA-reads the
            # neighbours' probe blocks through the mappings), so a transport
            # that faults or misreads costs a fallback to NCCL, not the run
            blobs, ok = [None] * world, [None] * world
            try:
                blob = mesh.peer_export()
            except dfg.DfgError:
                blob = None
            dist.all_gather_object(blobs, blob)
            lo_b = blobs[rank - 1] if rank > 0 else None
            hi_b = blobs[rank + 1] if rank < world - 1 else None
            linked = False
            if all(b is not None for b in blobs):
                good, detail = True, "forced (--halo peer)"
                if args.halo == "auto":
                    good, detail = dfg.probe_peer_transport([lo_b, hi_b], local)
                probe = {"rank": rank, "ok": good, "detail": detail}
                if good:
                    try:
                        mesh.link_peers(lo_b, hi_b)
                        linked = True
                    except dfg.DfgError as e:
                        probe["detail"] = f"link refused: {e}"
            dist.all_gather_object(ok, (linked, probe))
            probe = [p for _, p in ok]
            if all(lk for lk, _ in ok):
                halo = "peer"
            elif linked:
                mesh.link_peers(None, None)
        if halo == "nccl":
            uid = [dfg.dfg_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            dfg.dfg_mesh_init_comm(mesh.handle, uid[0], rank, world)
    plan = dfg.Plan(mesh, QCRIT, "fused").set_timing(2)   # kernel events inside the timed region
    out = torch.empty((nzl, n, n), dtype=torch.float32, device="cuda")
    stream = torch.cuda.Stream()
    cells_rank = nzl * n * n

    def barrier():
        if world > 1:
            dist.barrier()

    with torch.cuda.stream(stream):
        for _ in range(W):
            plan.execute(out, stream=stream)
    stream.synchronize()
    plan.reset_stats()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        e0.record(stream)
        for _ in range(K):
            plan.execute(out, stream=stream)
        e1.record(stream)
        e1.synchronize()
    torch.cuda.synchronize()
    barrier()
    ms = e0.elapsed_time(e1)
    st = plan.stats()
    # fused-kernel time per step: one launch at N=1; at N>1 the interior launch
    # plus the one or two boundary-plane launches that follow the halo exchange
    launches_per_step = st["kernel_count"] / max(1, K)
    kern_ms = st["kernel_ms_sum"] / max(1, st["kernel_launches_timed"]) * launches_per_step
    kern_ms_rank, ms_rank = kern_ms, ms
    t = torch.tensor([ms, kern_ms], device="cuda", dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms, kern_ms = float(t[0]), float(t[1])
    ms_step = ms / K
    value = n * n * NZ / (ms_step * 1e-3)          # every cell of the job once per step
    info = plan.info()

    # context for the roofline: a plain device copy (torch copy_, 4 GiB read +
    # 4 GiB written) back to back for ~1 s, i.e. HBM bandwidth under the same
    # board power cap a long step runs in (MEASURED_PEAKS is a burst figure)
    sustained = None
    if world == 1 and not args.no_strategies:
        a = torch.empty(1 << 30, dtype=torch.float32, device="cuda")
        b = torch.empty_like(a)
        b.copy_(a)
        torch.cuda.synchronize()
        reps = max(10, int(1.0 / (kern_ms * 1e-3 * 2.6)))
        with ClockSampler(local) as cclk:
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            c0.record()
            for _ in range(reps):
                b.copy_(a)
            c1.record()
            c1.synchronize()
        sustained = {"gb_per_s": 2 * a.numel() * 4 * reps / (c0.elapsed_time(c1) * 1e-3) / 1e9,
                     "reps": reps, "clocks": cclk.summary(),
                     "how": "torch copy_ of 4 GiB fp32, back to back, CUDA events (read + write bytes)"}
        del a, b
        torch.cuda.empty_cache()

    # burst and sustained side by side: the timed region above is K steps
    # (the driver's K = 20 is ~60 ms, too short for the 1 kW cap to engage);
    # 300 back-to-back steps of the same plan show the power-capped regime
    sustained_steps = None
    if world == 1 and not args.no_strategies and K < 300:
        n_s = 300
        plan.reset_stats()
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ClockSampler(local) as sclk:
            s0.record(stream)
            for _ in range(n_s):
                plan.execute(out, stream=stream)
            s1.record(stream)
            s1.synchronize()
        sst = plan.stats()
        s_kms = sst["kernel_ms_sum"] / max(1, sst["kernel_launches_timed"])
        sustained_steps = {"steps": n_s, "ms_per_step": s0.elapsed_time(s1) / n_s, "kernel_ms": s_kms,
                           "achieved_gb_per_s": ALGO_BYTES_PER_CELL * cells_rank / (s_kms * 1e-3) / 1e9,
                           "clocks": sclk.summary()}

    # roofline of the dominant kernel (the only kernel of the step)
    peak, peak_src = _peak()
    achieved = ALGO_BYTES_PER_CELL * cells_rank / (kern_ms * 1e-3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            tj = json.load(open(tp))
            if tj.get("n") == n:
                traffic = tj.get("dram_bytes_per_launch")
        except Exception:
            pass

    # e2e through the C ABI with host buffers (N = 1: host-pointer binding,
    # the library uploads inputs and downloads the result inside dfg_execute)
    e2e = None
    if world == 1:
        hostf = {c: fields[c].cpu().pin_memory() for c in "uvw"}
        hout = torch.empty((nzl, n, n), dtype=torch.float32).pin_memory()
        hmesh = dfg.Mesh(x, y, z)
        for c in "uvw":
            hmesh.bind(c, hostf[c], on_device=False)
        # the streamed strategy: z-chunks through a device ring, uploads /
        # kernel / downloads overlapped (fused with host buffers = serial)
        hplan = dfg.Plan(hmesh, QCRIT, "streamed")
        hplan.execute(hout, out_on_device=False)
        reps = 3
        t0 = time.perf_counter()
        for _ in range(reps):
            hplan.execute(hout, out_on_device=False)
        te = (time.perf_counter() - t0) / reps
        hs = hplan.stats()
        ok = bool(torch.equal(hout, out.cpu()))
        e2e = {"value": cells_rank / te, "unit": "cells/s",
               "h2d_bytes_per_step": hs["h2d_bytes"] // hs["executes"],
               "d2h_bytes_per_step": hs["d2h_bytes"] // hs["executes"],
               "ms_per_step": te * 1e3, "matches_device_result": ok, "strategy": "streamed",
               "pcie_gb_per_s": (hs["h2d_bytes"] + hs["d2h_bytes"]) / hs["executes"] / te / 1e9}
        # the PCIe bound of this leg: pinned copies alone (CUDA events), inputs
        # up and the result down overlapping (full duplex)
        scratch = torch.empty_like(fields["u"])
        bw = {}
        for name, dst, src in (("h2d", scratch, hostf["u"]), ("d2h", hout, out)):
            dst.copy_(src, non_blocking=True)
            torch.cuda.synchronize()
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            c0.record()
            for _ in range(3):
                dst.copy_(src, non_blocking=True)
            c1.record()
            c1.synchronize()
            bw[name] = 3 * src.numel() * src.element_size() / (c0.elapsed_time(c1) * 1e-3) / 1e9
        del scratch
        bound_s = max(e2e["h2d_bytes_per_step"] / (bw["h2d"] * 1e9), e2e["d2h_bytes_per_step"] / (bw["d2h"] * 1e9))
        e2e["pcie_bound"] = {"h2d_gb_per_s": bw["h2d"], "d2h_gb_per_s": bw["d2h"], "bound_ms": bound_s * 1e3,
                             "frac": bound_s / te,
                             "how": "pinned torch copies of 4 GiB alone; bound = max(h2d bytes / h2d rate, "
                                    "d2h bytes / d2h rate), i.e. full-duplex overlap"}
        hplan.close()
        hmesh.close()
        del hostf, hout
    else:
        # multi-GPU: pinned host -> device copies + dfg_execute + result read-back per step
        hostf = {c: fields[c].cpu().pin_memory() for c in "uvw"}
        hout = torch.empty((nzl, n, n), dtype=torch.float32).pin_memory()
        barrier()
        torch.cuda.synchronize()
        reps = 3
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        h0.record(stream)
        for _ in range(reps):
            with torch.cuda.stream(stream):
                for c in "uvw":
                    fields[c][g:g + nzl].copy_(hostf[c][g:g + nzl], non_blocking=True)
                plan.execute(out, stream=stream)
                hout.copy_(out, non_blocking=True)
        h1.record(stream)
        h1.synchronize()
        te = torch.tensor([h0.elapsed_time(h1) * 1e-3 / reps], dtype=torch.float64, device="cuda")
        dist.all_reduce(te, op=dist.ReduceOp.MAX)        # device time, max over ranks
        te = float(te[0])
        e2e = {"value": cells_rank * world / te, "unit": "cells/s",
               "h2d_bytes_per_step": 3 * nzl * n * n * 4 * world,
               "d2h_bytes_per_step": out.numel() * 4 * world, "ms_per_step": te * 1e3,
               "timing": "CUDA events on the step stream, max over ranks"}

    multi = None
    if world > 1:
        # per-rank halo bytes, kernel time and step time; max over ranks
        hm = mesh.halo_map()
        per = torch.tensor([st["halo_bytes"] / max(1, K), kern_ms_rank, ms_rank / K, launches_per_step, dist.get_world_size(), dist.get_rank(),
                            (ALGO_BYTES_PER_CELL * cells_rank / (kern_ms_rank * 1e-3) / 1e9), hm[1]],
                           dtype=torch.float64, device="cuda")
        allr = [torch.zeros_like(per) for _ in range(world)]
        dist.all_gather(allr, per)
        rows = [r.tolist() for r in allr]
        multi = {"halo_bytes_per_step": [int(r[0]) for r in rows],
                 "kernel_ms_per_step": [r[1] for r in rows],
                 "step_ms": [r[2] for r in rows],
                 "launches_per_step": [r[3] for r in rows],
                 "comm_rank_of_rank": [int(r[5]) for r in rows],
                 "comm_ranks": [int(r[4]) for r in rows],
                 "nccl_comm_ranks": [int(r[7]) for r in rows],
                 "comm": "comm_ranks: torch process group size seen by each rank; nccl_comm_ranks: libdfg's own "
                         "NCCL communicator (1 = none: the peer halo needs no communicator)",
                 "world_size": world,
                 "achieved_gb_per_s_per_rank": [r[6] for r in rows],
                 "roofline_frac_per_rank": [r[6] / _peak()[0] for r in rows],
                 "halo_mode": halo,
                 "halo_probe": probe,
                 "halo": ("peer memory: the boundary-plane launches read the neighbours' first/last owned "
                          "planes of u, v, w in place (CUDA IPC mappings, NVLink), after the interior planes; "
                          "step flags by stream write/wait-value" if halo == "peer" else
                          "NCCL send/recv of the first/last owned plane of u, v, w on a side stream, "
                          "overlapped with the interior planes; boundary planes launched after it")}

    strategies = variants = sweep = blocks = None
    if rank == 0 and world == 1 and not args.no_strategies:
        variants = variant_leg(dfg, mesh, out, QCRIT, torch, n)
        strategies = strategy_sweep(dfg, synth, torch, (e2e or {}).get("pcie_bound"))
        sweep = complexity_sweep(dfg, synth, torch)
        blocks = blocks_leg(torch)

    cpu = None
    if world > 1 and not args.no_cpu_baseline:
        cpu = slab_boundary_parity(dist, torch, rank, world, fields, out, x, y, z, n, nzl, g)
        barrier()
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        same = n == N1 and world == 1
        cpu = cpu_baseline_leg(gpu_out=out if same else None, gpu_fields=fields if same else None)
        if not args.no_cpu_mt:
            try:
                cpu["oracle_mt"] = cpu_baseline_mt()
            except Exception as e:  # a host without multiprocessing support
                cpu["oracle_mt"] = {"unavailable": repr(e)[:200]}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "cells/s", "n_gpus": world, "steps": K, "warmup": W,
            "ms_per_step": ms_step, "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
            "dtype": "f32", "data": "synthetic",
            "config": {"workload": (f"fused Q-criterion, {n}^3 fp32 rectilinear mesh per GPU " if args.scaling == "weak"
                                    else f"fused Q-criterion, one {n}^3 fp32 rectilinear mesh over {world} GPU(s) ")
                                   + f"(mesh {n}x{n}x{NZ}, z-slabs + 1-plane halo when N>1: " + (halo or "none") + ")",
                       "expression": "qcrit (Fig. 3C completed)", "strategy": "fused",
                       "cells_per_gpu": cells_rank, "fused_kernel": {1: "tma", 2: "general", 3: "pointwise", 5: "tile"}.get(
                           info["variant"]), "regs": info["regs"],
                       "arithmetic": "exact: every cell bit-identical to the fp32 oracle (two-operation grad3d quotient "
                                     f"on verified axes, mask {info.get('div2_axes')}); the within-tolerance 'fast' "
                                     "quotient and the hand-written reference kernel are under 'variants'",
                       "l2": f"inputs {3 * cells_rank * 4 / 1e9:.1f} GB per GPU >> 126 MB L2; no flush needed",
                       "parallelism": f"zslab{world}",
                       **({"one_gpu_functional_test": True} if one_gpu else {})},
            "hbm_gbs": ALGO_BYTES_PER_CELL * cells_rank * world / (ms_step * 1e-3) / 1e9 / world,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                         "kernel": "dfg_fused_tma", "kernel_ms": kern_ms,
                         "algorithmic_bytes_per_launch": ALGO_BYTES_PER_CELL * cells_rank,
                         **({"sustained_copy": sustained, "frac_of_sustained_copy": achieved / sustained["gb_per_s"]}
                            if sustained else {}),
                         **({"sustained_300_steps": dict(sustained_steps,
                                                         frac=sustained_steps["achieved_gb_per_s"] / peak,
                                                         frac_of_sustained_copy=(sustained_steps["achieved_gb_per_s"] /
                                                                                 sustained["gb_per_s"]
                                                                                 if sustained else None))}
                            if sustained_steps else {})},
            "e2e": e2e,
            "multi_gpu": multi,
            "gpu_launches": st["kernel_count"],
            "clocks": clk.summary(),
            "frac_of_spec_8tbs": achieved / 8000.0,
            "variants": variants,
            "strategies": strategies,
            "complexity_sweep_768": sweep,
            "visit_blocks": blocks,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    # release the library's NCCL communicator before torch tears its own down
    torch.cuda.synchronize()
    plan.close()
    mesh.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _time_plan(plan, out, torch, iters):
    plan.set_timing(2)
    for _ in range(3):
        plan.execute(out)
    torch.cuda.synchronize()
    plan.reset_stats()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters):
        plan.execute(out)
    e1.record()
    e1.synchronize()
    st = plan.stats()
    return e0.elapsed_time(e1) / iters, st["kernel_ms_sum"] / max(1, st["kernel_launches_timed"])


def variant_leg(dfg, mesh, out_exact, src, torch, n):
    """The division variants of the fused kernel on the bench inputs (context:
    the headline uses the exact variant).  'fast' = num * (1/d): one rounding
    more per derivative, not bit-identical to the oracle."""
    res = {}
    for var in ("fast",):
        os.environ["DFG_FUSED_VARIANT"] = var
        try:
            plan = dfg.Plan(mesh, src, "fused")
        finally:
            os.environ.pop("DFG_FUSED_VARIANT", None)
        out = torch.empty_like(out_exact)
        ms, kms = _time_plan(plan, out, torch, 50)
        diff = (out - out_exact).abs().max().item() / out_exact.abs().max().item()
        res[var] = {"kernel_ms": kms, "cells_per_s": n ** 3 / (kms * 1e-3),
                    "algorithmic_gb_per_s": ALGO_BYTES_PER_CELL * n ** 3 / (kms * 1e-3) / 1e9,
                    "normwise_diff_vs_exact": diff, "bit_identical": bool(torch.equal(out, out_exact))}
        plan.close()
        del out
    # the hand-written reference kernel (L243; strategy "reference")
    plan = dfg.Plan(mesh, "qcrit", "reference")
    out = torch.empty_like(out_exact)
    ms, kms = _time_plan(plan, out, torch, 50)
    diff = (out - out_exact).abs().max().item() / out_exact.abs().max().item()
    res["reference_kernel"] = {"kernel_ms": kms, "cells_per_s": n ** 3 / (kms * 1e-3),
                               "algorithmic_gb_per_s": ALGO_BYTES_PER_CELL * n ** 3 / (kms * 1e-3) / 1e9,
                               "normwise_diff_vs_exact": diff}
    plan.close()
    del out
    return res


def blocks_leg(torch):
    """the paper's VisIt decomposition (Fig. 7,
    L315: blocks of 192 x 192 x 256 with ghost shells, 12 sub-grids per GPU)
    -- one plan per block back to back vs all blocks of the device in one
    persistent launch (TMA kernel on 16-byte padded shells, cp.async ring on
    packed shells) vs one mesh of the same cells; 16 algorithmic B / cell."""
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    import blocks_overhead
    res = {}
    for pad, name in ((1, "padded_shells"), (0, "packed_shells")):
        r = blocks_overhead.measure(12, 192, 192, 256, pad)
        r["algorithmic_gb_per_s_one_launch"] = ALGO_BYTES_PER_CELL * r["cells"] / (r["ms_batched"] * 1e-3) / 1e9
        res[name] = r
        torch.cuda.empty_cache()
    return res


ORACLE_CHECKS = True   # bench.py --no-cpu-baseline: no oracle use at all


def _window_parity(src, names, dt, fields, out, x, y, z, n):
    """Sampled full-size parity of a sweep case: the oracle on three windows
    of the GPU's own inputs (the low corner with the global one-sided
    boundaries, an interior block, the high corner), full rows in x, compared
    bit for bit with the fused kernel's output over the window cells whose
    stencil lies inside the window (oracle.evaluate's valid mask)."""
    if not ORACLE_CHECKS:
        return None
    from oracle import evaluate as oev
    from oracle.lang import build_dag
    dag = build_dag(src, tuple(names), dt)
    u = np.uint32 if dt == "f32" else np.uint64
    cells = bad = 0
    for k0, j0 in ((0, 0), (n // 2 - 3, n // 2 - 4), (n - 6, n - 8)):
        win = {nm: fields[c][k0:k0 + 6, j0:j0 + 8, :].cpu().numpy() for nm, c in zip(names, "uvw")}
        ref, valid = oev.evaluate(dag, win, oev.MeshWindow(x, y, z, i0=0, j0=j0, k0=k0))
        got = out[k0:k0 + 6, j0:j0 + 8, :].cpu().numpy()
        cells += int(valid.sum())
        bad += int(np.count_nonzero(got[valid].view(u) != ref[valid].view(u)))
    return {"cells_compared": cells, "mismatches": bad, "windows": "6 planes x 8 rows x all columns at the low "
            "corner, the centre and the high corner"}


def complexity_sweep(dfg, synth, torch):
    """Config 5: the expression-complexity sweep (intro -> VelMag -> VortMag
    -> Q) at 768^3, fp32 and fp64, fused strategy, device-resident inputs."""
    PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}
    n = 768
    res = {}
    for dt, tt, npt in (("f32", torch.float32, np.float32), ("f64", torch.float64, np.float64)):
        x, y, z = synth.rt_coords(n, n, n, npt)
        x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
        fields = {c: synth.rt_velocity(c, x64, y64, z64, None, tt, "cuda") for c in "uvw"}
        out = torch.empty((n, n, n), dtype=tt, device="cuda")
        for name in ("intro", "velmag", "vortmag", "qcrit"):
            src, names = PAPER_PROGRAMS[name]
            mesh = dfg.Mesh(x, y, z)
            for nm, c in zip(names, "uvw"):
                mesh.bind(nm, fields[c])
            plan = dfg.Plan(mesh, src, "fused")
            ms, kms = _time_plan(plan, out, torch, 20)
            nbytes = (len(names) + 1) * np.dtype(npt).itemsize
            info = plan.info()
            res[f"{name}_{dt}"] = {"filters": info["filters"], "kernel_ms": kms, "cells_per_s": n ** 3 / (kms * 1e-3),
                                   "algorithmic_gb_per_s": nbytes * n ** 3 / (kms * 1e-3) / 1e9,
                                   "bytes_per_cell": nbytes, "regs": info["regs"],
                                   "kernel": {1: "tma", 2: "general", 3: "pointwise", 5: "tile"}.get(info["variant"]),
                                   "oracle_parity": _window_parity(src, names, dt, fields, out, x, y, z, n)}
            plan.close()
            mesh.close()
        del fields, out
        torch.cuda.empty_cache()
    return res


def strategy_sweep(dfg, synth, torch, pcie=None):
    """Config 1 (32^3 VortMag, the three strategies: launch-bound), config 2
    (192^3: fused vs staged vs roundtrip, VelMag / VortMag / Q) and config 3
    (512^3 Q: staged under device-memory caps vs fused)."""
    PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}
    out = {"config1_32_vortmag": _strategies_at(dfg, synth, torch, 32, PAPER_PROGRAMS["vortmag"][0],
                                                ("fused", "staged", "roundtrip"), 7, pcie),
           "config2_192": {}}
    for name in ("velmag", "vortmag", "qcrit"):
        out["config2_192"][name] = _strategies_at(dfg, synth, torch, 192, PAPER_PROGRAMS[name][0],
                                                  ("fused", "staged", "roundtrip"), 7, pcie)
    GiB = 1 << 30
    c3 = _strategies_at(dfg, synth, torch, 512, PAPER_PROGRAMS["qcrit"][0], ("fused", "staged"), 3)
    # staged under device-memory caps: the paper's list order fails below its
    # footprint (L309); the memory-aware order (NEXT #3) runs down to its own
    caps = {}
    n3 = 512
    x, y, z = synth.rt_coords(n3, n3, n3, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    flds = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, t in flds.items():
        mesh.bind(c, t)
    q = PAPER_PROGRAMS["qcrit"][0]
    ref = torch.empty((n3, n3, n3), device="cuda")
    dfg.Plan(mesh, q, "fused").execute(ref)
    o = torch.empty_like(ref)
    for cap_gib in (16, 12, 10, 8, 4):
        try:
            p = dfg.Plan(mesh, q, "staged", cap_gib * GiB)
            sched = p.schedule()
            ms, _ = _time_plan(p, o, torch, 2)
            caps[f"{cap_gib}GiB"] = {"runs": True, "order": "list" if sched == sorted(sched) else "memory-aware",
                                     "highwater_gib": p.stats()["dev_highwater_bytes"] / GiB, "ms": ms,
                                     "bit_identical_to_fused": bool(torch.equal(o, ref))}
            p.close()
        except dfg.DfgError as e:
            caps[f"{cap_gib}GiB"] = {"runs": False, "error": e.name}
    # hybrid (NEXT #3 spill-to-host): the caps staged cannot meet, intermediates
    # spill to pinned host memory (device-resident inputs and output)
    hyb = {}
    for cap_gib in (8, 6, 4):
        try:
            p = dfg.Plan(mesh, q, "hybrid", cap_gib * GiB)
            ms, _ = _time_plan(p, o, torch, 2)
            st = p.stats()
            ex = max(1, st["executes"])
            hyb[f"{cap_gib}GiB"] = {"runs": True, "ms": ms, "highwater_gib": st["dev_highwater_bytes"] / GiB,
                                    "spills_per_execute": st["d2h_count"] // ex,
                                    "reloads_per_execute": st["h2d_count"] // ex,
                                    "pcie_gib_per_execute": (st["h2d_bytes"] + st["d2h_bytes"]) / ex / GiB,
                                    "bit_identical_to_fused": bool(torch.equal(o, ref))}
            p.close()
        except dfg.DfgError as e:
            hyb[f"{cap_gib}GiB"] = {"runs": False, "error": e.name}
    del flds, ref, o
    torch.cuda.empty_cache()
    c3["staged_caps"] = caps
    c3["hybrid_caps"] = hyb
    out["config3_512_qcrit"] = c3
    return out


def _strategies_at(dfg, synth, torch, n, src, strategies, runs, pcie=None):
    x, y, z = synth.rt_coords(n, n, n, np.float32)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    mesh = dfg.Mesh(x, y, z)
    bufs = {c: synth.rt_velocity(c, x64, y64, z64, None, torch.float32, "cuda") for c in "uvw"}
    for c, b in bufs.items():
        mesh.bind(c, b)
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    clean = torch.ones(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    res = {}
    ref = None
    for s in strategies:
        plan = dfg.Plan(mesh, src, s).set_timing(0)   # no library events inside the timed interval
        out = torch.empty((n, n, n), dtype=torch.float32, device="cuda")
        for _ in range(2):
            plan.execute(out)
        torch.cuda.synchronize()
        times = []
        for _ in range(runs):               # the paper's protocol: 7 runs, drop min/max (L241)
            flush.zero_()                   # L2 flush (working set < 4x L2) ...
            clean.sum()                     # ... then read 512 MB: L2 cold AND clean (no write-back of
            torch.cuda.synchronize()        # the flush buffer lands inside the timed execute)
            torch.cuda._sleep(2_000_000)    # ~1 ms of device work: the execute is enqueued behind it,
            #                                 so host-side launch latency is not part of the interval
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.execute(out)
            e1.record()
            e1.synchronize()
            times.append(e0.elapsed_time(e1))
        times = sorted(times)[1:-1]
        ms = sum(times) / len(times)
        st = plan.stats()
        ex = st["executes"]
        # staged / roundtrip move their intermediates through device memory;
        # when one problem array (4 B x n^3) fits the 126 MB L2 those round
        # trips stay on chip, so the figure is device-memory-system traffic,
        # not HBM bandwidth (config 2: 28 MB arrays)
        l2_resident = 4 * n ** 3 * 4 <= 126e6 and s != "fused"
        res[s] = {"cells_per_s": n ** 3 / (ms * 1e-3), "ms": ms,
                  ("device_gb_per_s_l2_resident" if l2_resident else "device_gb_per_s"):
                      st["predicted_hbm_bytes"] / (ms * 1e-3) / 1e9,
                  "predicted_device_bytes": st["predicted_hbm_bytes"],
                  "pcie_bytes": (st["h2d_bytes"] + st["d2h_bytes"]) // ex,
                  **({"pcie_bound_ms": 1e3 * (st["h2d_bytes"] / ex / (pcie["h2d_gb_per_s"] * 1e9)
                                              + st["d2h_bytes"] / ex / (pcie["d2h_gb_per_s"] * 1e9)),
                      "pcie_bound_how": "h2d bytes / pinned h2d rate + d2h bytes / pinned d2h rate (the "
                                        "roundtrip's transfers are serial: every filter waits for its result)"}
                     if pcie and st["h2d_bytes"] + st["d2h_bytes"] > 0 else {}),
                  "kernels_per_execute": st["kernel_count"] // ex,
                  "highwater_bytes": st["dev_highwater_bytes"]}
        if ref is None:
            ref = out.clone()
            res[s]["oracle_parity"] = _window_parity(src, ("u", "v", "w"), "f32", bufs, out, x, y, z, n)
        else:
            res[s]["bit_identical_to_fused"] = bool(torch.equal(ref, out))
        plan.close()
        del out
    del bufs, flush, clean
    torch.cuda.empty_cache()
    return {"workload": f"{n}^3 fp32, device-resident inputs, L2 flushed (512 MB write + 512 MB read), "
                        f"device time of one execute (enqueued behind a device sleep), trimmed mean of {runs} runs",
            **res}


if __name__ == "__main__":
    sys.exit(main())
