"""Exercise the peer-memory z-slab halo with G ranks on ONE GPU (developer tool).

    python tools/peer_ranks.py [--ranks 2] [--n 64] [--nz 40] [--steps 3]

Each rank is its own process (torch.multiprocessing spawn) with a z-slab of
the RT-like mesh on cuda:0; gloo is used for plumbing only.  Every rank
exports its slab (dfg_mesh_peer_export: CUDA IPC handles of its fields and of
its step flags), the blobs are all-gathered, and every rank links the slabs
directly below and above (dfg_mesh_link_peers).  Then each rank runs `steps`
time steps: it rewrites its owned planes (fields x (1 + t)) on the stream
and executes the fused plan -- the kernel reads the neighbours' boundary
planes in place through the IPC mappings, ordered by the step flags (stream
memory operations).  Same code as the NVLink case; only the mappings are
same-device.  Rank 0 compares every step's stitched slabs with the
single-slab result of that step's fields bit for bit and prints one JSON line.
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
                       "WORLD_SIZE": str(world)})
    if args.kernel:
        os.environ["DFG_FUSED_KERNEL"] = args.kernel
    import torch
    import torch.distributed as dist

    import paper_conf_sc_harrisonnmjc12_b200 as dfg
    import synth
    PAPER_PROGRAMS = {k: (dfg.paper_program(k), dfg.PAPER_INPUTS[k]) for k in dfg.PAPER_INPUTS}

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    nx, n, NZ = args.nx or args.n, args.n, args.nz
    T, tt = (np.float32, torch.float32) if args.dtype == "f32" else (np.float64, torch.float64)
    x, y, z = synth.rt_coords(nx, n, NZ, T)
    x64, y64, z64 = (a.astype(np.float64) for a in (x, y, z))
    k0, nzl = dfg.dfg_partition(NZ, world, rank)
    src, names = PAPER_PROGRAMS[args.prog]
    recipe = dict(zip(names, "uvw"))
    base = {name: synth.rt_velocity(c, x64, y64, z64, (k0, k0 + nzl, 0, n, 0, nx), tt, "cuda")
            for name, c in recipe.items()}
    # ghost planes stay NaN: the peer path must never read them
    fields = {name: torch.full((nzl + 2, n, nx), float("nan"), dtype=tt, device="cuda") for name in recipe}
    mesh = dfg.Mesh(x, y, z, nz_local=nzl, z_offset=k0, ghost=1)
    for c, b in fields.items():
        mesh.bind(c, b)
    blobs = [None] * world
    dist.all_gather_object(blobs, mesh.peer_export())
    mesh.link_peers(blobs[rank - 1] if rank > 0 else None, blobs[rank + 1] if rank < world - 1 else None)
    plan = dfg.Plan(mesh, src, "fused")
    outs = []
    for t in range(args.steps):
        for name in recipe:
            fields[name][1:1 + nzl].copy_(base[name] * (1 + t))   # this step's fields, on the stream
        out = torch.empty((nzl, n, nx), dtype=tt, device="cuda")
        plan.execute(out, stream=torch.cuda.current_stream())
        outs.append(out)
    torch.cuda.synchronize()
    st = plan.stats()
    info = plan.info()
    got = [o.cpu().numpy() for o in outs]
    ghosts_untouched = all(bool(torch.isnan(b[0]).all() and torch.isnan(b[nzl + 1]).all()) for b in fields.values())
    parts = [None] * world
    dist.all_gather_object(parts, (rank, k0, nzl, got, st["halo_bytes"], st["kernel_count"], info["halo"],
                                   ghosts_untouched))
    ok = None
    if rank == 0:
        whole_mesh = dfg.Mesh(x, y, z)
        wbase = {name: synth.rt_velocity(c, x64, y64, z64, None, tt, "cuda") for name, c in recipe.items()}
        wf = {name: torch.empty_like(b) for name, b in wbase.items()}
        for c, b in wf.items():
            whole_mesh.bind(c, b)
        wplan = dfg.Plan(whole_mesh, src, "fused")
        from oracle import evaluate as oev
        from oracle.lang import build_dag
        dag = build_dag(src, tuple(recipe), args.dtype)
        ok = oracle_ok = True
        for t in range(args.steps):
            for name in recipe:
                wf[name].copy_(wbase[name] * (1 + t))
            wout = torch.empty((NZ, n, nx), dtype=tt, device="cuda")
            wplan.execute(wout)
            torch.cuda.synchronize()
            stitched = np.concatenate([p[3][t] for p in sorted(parts, key=lambda p: p[1])])
            ok = ok and bool(np.array_equal(stitched, wout.cpu().numpy()))
            # and against the oracle on the same step's arrays
            want = oev.evaluate_full(dag, {k: v.cpu().numpy() for k, v in wf.items()}, x, y, z)
            oracle_ok = oracle_ok and bool(np.array_equal(stitched, want))
        ok = ok and oracle_ok
        pb = n * nx * np.dtype(T).itemsize
        per = [p[4] / (args.steps * pb * ((p[0] > 0) + (p[0] < world - 1))) for p in parts]
        print(json.dumps({"ranks": world, "nx": nx, "n": n, "nz": NZ, "prog": args.prog, "dtype": args.dtype,
                          "steps": args.steps, "bit_identical_to_single_slab": ok,
                          "bit_identical_to_oracle": oracle_ok,
                          "halo_fields": per[0], "halo_modes": [p[6] for p in parts],
                          "ghost_planes_untouched": [p[7] for p in parts],
                          "kernels_per_execute": [p[5] / args.steps for p in parts],
                          "transport": "CUDA IPC mappings on one GPU (NVLink peers on a multi-GPU node)"}),
              flush=True)
    dist.barrier()
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
    ap.add_argument("--nx", type=int, default=0, help="x cells (default: --n)")
    ap.add_argument("--nz", type=int, default=40)
    ap.add_argument("--prog", default="qcrit")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--dtype", default="f32", choices=["f32", "f64"])
    ap.add_argument("--kernel", default="", help="DFG_FUSED_KERNEL for every rank (e.g. tile)")
    ap.add_argument("--as-rank", type=int, default=-1,
                    help="run only this rank in this process (start every rank yourself, same --port), "
                         "e.g. each under compute-sanitizer")
    ap.add_argument("--port", type=int, default=0)
    args = ap.parse_args()
    port = args.port or 29500 + (os.getpid() % 2000)
    if args.as_rank >= 0:
        worker(args.as_rank, args.ranks, args, port)
        return
    import torch.multiprocessing as mp
    mp.spawn(worker, args=(args.ranks, args, port), nprocs=args.ranks, join=True)


if __name__ == "__main__":
    main()
