"""Exercise the NCCL z-slab path with G ranks on ONE GPU (developer tool).

    python tools/nccl_two_ranks.py [--ranks 2] [--n 64] [--nz 40] [--overlap 1]

NCCL refuses two ranks on one device within a host, so each rank gets its own
NCCL_HOSTID: NCCL then treats them as separate hosts and moves the halo
planes over its socket transport (loopback).  That exercises exactly the
library's multi-GPU code: dfg_nccl_unique_id, dfg_mesh_init_comm, the NCCL
group send/recv of the ghost planes (on the plan's side stream, overlapped
with the interior planes) and the boundary-plane launches -- only the
transport differs from NVLink.  Rank 0 compares the stitched slab results
with the single-slab result bit for bit and prints one JSON line.
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def worker(rank, world, args, port):
    os.environ.update({"MASTER_ADDR": "127.0.0.1", "MASTER_PORT": str(port), "RANK": str(rank),
                       "WORLD_SIZE": str(world), "NCCL_HOSTID": f"dfg-rank-{rank}", "NCCL_SOCKET_IFNAME": "lo",
                       "NCCL_IB_DISABLE": "1", "NCCL_P2P_DISABLE": "1", "NCCL_SHM_DISABLE": "1",
                       "DFG_HALO_OVERLAP": str(args.overlap)})
    import torch
    import torch.distributed as dist

    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    import synth
    PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)  # plumbing only: the halo is the library's NCCL
    n, NZ = args.n, args.nz
    T, tt = (np.float32, torch.float32) if args.dtype == "f32" else (np.float64, torch.float64)
    x, y, z = synth.rt_coords(n, n, NZ, T)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    k0, nzl = dfg.dfg_partition(NZ, world, rank)
    src, names = PAPER_PROGRAMS[args.prog]
    recipe = dict(zip(names, "uvw"))            # intro: b = u-recipe, c = v-recipe
    fields = {}
    for name, c in recipe.items():
        buf = torch.zeros((nzl + 2, n, n), dtype=tt, device="cuda")
        buf[1:1 + nzl] = synth.rt_velocity(c, x64, y64, z64, (k0, k0 + nzl, 0, n, 0, n), tt, "cuda")
        fields[name] = buf
    mesh = dfg.Mesh(x, y, z, nz_local=nzl, z_offset=k0, ghost=1)
    for c, b in fields.items():
        mesh.bind(c, b)
    uid = [dfg.dfg_nccl_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(uid, src=0)
    dfg.dfg_mesh_init_comm(mesh.handle, uid[0], rank, world)
    plan = dfg.Plan(mesh, src, "fused")
    out = torch.empty((nzl, n, n), dtype=tt, device="cuda")
    for _ in range(args.reps):
        plan.execute(out)
    torch.cuda.synchronize()
    st = plan.stats()
    # ghost planes as received, for the check against the neighbours' owned planes
    got = out.cpu().numpy()
    parts = [None] * world
    dist.all_gather_object(parts, (rank, k0, nzl, got, st["halo_bytes"], st["kernel_count"]))
    ok = None
    if rank == 0:
        whole_mesh = dfg.Mesh(x, y, z)
        wf = {name: synth.rt_velocity(c, x64, y64, z64, None, tt, "cuda") for name, c in recipe.items()}
        for c, b in wf.items():
            whole_mesh.bind(c, b)
        wout = torch.empty((NZ, n, n), dtype=tt, device="cuda")
        dfg.Plan(whole_mesh, src, "fused").execute(wout)
        torch.cuda.synchronize()
        whole = wout.cpu().numpy()
        stitched = np.concatenate([p[3] for p in sorted(parts, key=lambda p: p[1])])
        from oracle import evaluate as oev
        from oracle.lang import build_dag
        want = oev.evaluate_full(build_dag(src, tuple(recipe), args.dtype),
                                 {k: v.cpu().numpy() for k, v in wf.items()}, x, y, z)
        oracle_ok = bool(np.array_equal(stitched, want))      # the oracle itself
        ok = bool(np.array_equal(stitched, whole)) and oracle_ok
        pb = n * n * np.dtype(T).itemsize
        # halo fields = the stencil inputs: the same whole number on every rank
        per = [p[4] / (args.reps * pb * ((p[0] > 0) + (p[0] < world - 1))) for p in parts]
        halo_ok = all(v == per[0] and v == int(v) and v >= 1 for v in per)
        print(json.dumps({"ranks": world, "n": n, "nz": NZ, "prog": args.prog, "dtype": args.dtype,
                          "overlap": args.overlap,
                          "bit_identical_to_single_slab": ok, "bit_identical_to_oracle": oracle_ok, "halo_bytes_ok": halo_ok, "halo_fields": per[0],
                          "kernels_per_execute": [p[5] / args.reps for p in parts],
                          "transport": "NCCL socket (loopback), one GPU, per-rank NCCL_HOSTID"}), flush=True)
    plan.close()
    mesh.close()
    dist.barrier()
    dist.destroy_process_group()
    if rank == 0 and not ok:
        sys.exit(1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=2)
    ap.add_argument("--n", type=int, default=64)
    ap.add_argument("--nz", type=int, default=40)
    ap.add_argument("--prog", default="qcrit")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--overlap", type=int, default=1)
    ap.add_argument("--dtype", default="f32", choices=["f32", "f64"])
    args = ap.parse_args()
    import torch.multiprocessing as mp
    port = 29500 + (os.getpid() % 2000)
    mp.spawn(worker, args=(args.ranks, args, port), nprocs=args.ranks, join=True)


if __name__ == "__main__":
    main()
