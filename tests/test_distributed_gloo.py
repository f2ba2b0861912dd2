"""World-size-2 (and 3) CPU tests of the z-slab decomposition with torch.distributed
over gloo: the partition (dfg_partition from libdfg), the unique-id broadcast
the bench performs, and the ghost-plane exchange pattern of
PlanImpl::halo_exchange (send the first owned plane to r-1 and the last to
r+1, receive into ghost planes 0 and nz_r+1) -- here with gloo send/recv of the
same planes, each rank evaluating its slab with the oracle.  The gathered
result must equal the single-process evaluation bit for bit."""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_sc_harrisonnmjc12_b200", "libdfg.so")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shape, prog, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sc_harrisonnmjc12_b200 as dfg
        import synth
        from oracle import evaluate as oev
        from oracle import halo as ohalo
        from oracle.lang import PAPER_PROGRAMS, build_dag

        nx, ny, NZ = shape
        k0, nzr = dfg.dfg_partition(NZ, world, rank)
        assert (k0, nzr) == ohalo.partition(NZ, world, rank)
        # the bench's unique-id broadcast (any 128 bytes will do on CPU)
        uid = [bytes(range(128)) if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        assert uid[0] == bytes(range(128))

        x, y, z, f = synth.rt_inputs(nx, ny, NZ, dtype=np.float32)
        names = PAPER_PROGRAMS[prog][1]
        fields = dict(zip(names, [f[c] for c in "uvw"]))
        # local buffers with one ghost plane per side; owned planes 1..nzr
        loc = {}
        for n, t in fields.items():
            b = torch.zeros((nzr + 2, ny, nx), dtype=torch.float32)
            b[1:nzr + 1] = t[k0:k0 + nzr]
            loc[n] = b
        m = ohalo.halo_map(NZ, k0, nzr, rank, world, nx, ny, 4)
        has_lo, has_hi = m[6], m[7]
        # halo exchange with the library's plane pattern
        for n in names:
            b = loc[n]
            reqs = []
            if has_lo:
                reqs.append(dist.isend(b[m[10]].contiguous(), m[8]))
            if has_hi:
                reqs.append(dist.isend(b[m[11]].contiguous(), m[9]))
            if has_lo:
                t = torch.empty((ny, nx))
                dist.recv(t, m[8])
                b[m[12]] = t
            if has_hi:
                t = torch.empty((ny, nx))
                dist.recv(t, m[9])
                b[m[13]] = t
            for r in reqs:
                r.wait()
        # evaluate the slab window (ghosts included where they exist)
        lo = 0 if has_lo else 1
        hi = nzr + 2 if has_hi else nzr + 1
        win = {n: loc[n][lo:hi].numpy() for n in names}
        dag = build_dag(PAPER_PROGRAMS[prog][0], names, "f32")
        res, valid = oev.evaluate(dag, win, oev.MeshWindow(x, y, z, k0=k0 - (1 if has_lo else 0)))
        own = res[(1 if has_lo else 0):(1 if has_lo else 0) + nzr]
        assert valid[(1 if has_lo else 0):(1 if has_lo else 0) + nzr].all()
        parts = [None] * world
        dist.all_gather_object(parts, (rank, own))
        if rank == 0:
            got = np.concatenate([p[1] for p in sorted(parts, key=lambda t: t[0])])
            whole = oev.evaluate_full(dag, {n: t.numpy() for n, t in fields.items()}, x, y, z)
            q.put(bool(np.array_equal(got, whole)))
    finally:
        dist.destroy_process_group()


@pytest.mark.skipif(not os.path.exists(LIB), reason="libdfg.so not built")
@pytest.mark.parametrize("world,shape,prog", [(2, (12, 10, 9), "qcrit"), (3, (8, 6, 10), "vortmag"),
                                              (2, (6, 5, 4), "intro")])
def test_zslab_halo_over_gloo(world, shape, prog):
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    mp.start_processes(_worker, args=(world, _free_port(), shape, prog, q), nprocs=world, join=True,
                       start_method="spawn")
    assert q.get() is True
