"""The N > 1 path's host logic on CPU (gloo, world_size 2 and 3): the slab partition
(csx_shard_rows) and the halo-exchange schedule (csx_halo_schedule) that csx_run_sharded feeds
to NCCL are executed here with torch.distributed send/recv on CPU tensors, with the ORACLE as
the per-slab compute engine.  The gathered slabs must equal the single-domain oracle.

Per pass of Tf steps each rank holds its slab plus r*Tf ghost rows on every side that has a
neighbour; running Tf plain steps on that padded slab corrupts only the ghost rows (the error
front moves r rows per step), so the interior is exact — the property the GPU path relies on.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, name, ext, T, bc, tf, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
        s = synth.SHAPES[name]
        w = synth.random_weights(name)
        plan = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=tf)
        tfm = plan.info()["fuse_steps"]
        h = s.radius * tfm
        lo, hi = plan.shard_rows(rank, world)
        sched = plan.halo_schedule(rank, world)
        local = synth.grid(ext, rows=(lo, hi)).copy()
        El = hi - lo
        has_up = any(k == "recv" and row < 0 for k, _, row, _ in sched)
        has_dn = any(k == "recv" and row >= El for k, _, row, _ in sched)
        done = 0
        while done < T:
            step = min(tfm, T - done)
            pad = np.zeros((El + 2 * h,) + tuple(ext[1:]))
            pad[h:h + El] = local
            # post the schedule in order (gloo send/recv are blocking: isend/irecv + wait)
            reqs = []
            for kind, peer, row, n in sched:
                buf = torch.from_numpy(np.ascontiguousarray(pad[h + row:h + row + n]))
                if kind == "send":
                    reqs.append((None, dist.isend(buf, peer)))
                else:
                    reqs.append(((row, n, buf), dist.irecv(buf, peer)))
            for meta, r in reqs:
                r.wait()
                if meta is not None:
                    row, n, buf = meta
                    pad[h + row:h + row + n] = buf.numpy()
            if bc == "fixed":
                # FIXED: a side without a neighbour is a global face (its frame is held by the
                # oracle); a side with one carries its r*Tf ghost rows
                start = 0 if has_up else h
                end = El + 2 * h if has_dn else El + h
                res = oracle.run(pad[start:end], w, "fixed", step)
                local = res[h - start:h - start + El]
            else:
                res = oracle.run(pad, w, "periodic", step)
                local = res[h:h + El]
            done += step
        gathered = [None] * world if rank == 0 else None
        dist.gather_object(local, gathered, dst=0)
        if rank == 0:
            full = np.concatenate(gathered, axis=0)
            ref = oracle.run(synth.grid(ext), w, bc, T)
            q.put(float(np.max(np.abs(full - ref)) / np.max(np.abs(ref))))
    except Exception as e:  # surface errors to the parent
        q.put(repr(e))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
@pytest.mark.parametrize("name,ext,T,tf", [("box2d9p", (61, 40), 7, 3), ("heat1d", (301,), 17, 7),
                                           ("heat3d", (14, 9, 10), 3, 1)])
def test_sharded_matches_single_domain(world, bc, name, ext, T, tf):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, ext, T, bc, tf, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
    assert not isinstance(res, str), res
    assert res <= 1e-13


def _pencil_worker(rank, world, port, p0, p1, name, ext, T, bc, tf, q):
    """Rank `rank` of a p0 x p1 pencil/block grid: csx_shard_box + csx_pencil_schedule executed
    with gloo isend/irecv on numpy blocks padded by h = r*Tf on both split axes; the oracle
    runs every pass on the padded block (FIXED: sides without a neighbour are global faces and
    are not padded)."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
        s = synth.SHAPES[name]
        w = synth.random_weights(name)
        plan = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=tf)
        tfm = plan.info()["fuse_steps"]
        h = s.radius * tfm
        lo, hi = plan.shard_box(rank, p0, p1)
        sched = plan.pencil_schedule(rank, p0, p1)
        full0 = synth.grid(ext)
        local = full0[tuple(slice(a, b) for a, b in zip(lo, hi))].copy()
        El = local.shape
        # split axes in numpy order: (0, 1) for both 2D (rows, cols) and 3D (z, y)
        has = {(ph, side): any(k == "recv" and p == ph and ((row < 0) if side == 0 else (row >= El[1 - ph]))
                               for p, k, _, row, _ in sched)
               for ph in (0, 1) for side in (0, 1)}
        done = 0
        while done < T:
            step = min(tfm, T - done)
            pad = np.zeros((El[0] + 2 * h, El[1] + 2 * h) + tuple(El[2:]))
            pad[h:h + El[0], h:h + El[1]] = local
            for phase in (0, 1):
                reqs = []
                selfq = []  # a 1-wide PERIODIC axis talks to itself: k-th send -> k-th recv
                for ph, kind, peer, row, n in sched:
                    if ph != phase:
                        continue
                    if phase == 0:   # second split axis, owned range of the first
                        idx = (slice(h, h + El[0]), slice(h + row, h + row + n))
                    else:            # first split axis, full padded second axis (corners)
                        idx = (slice(h + row, h + row + n),)
                    buf = torch.from_numpy(np.ascontiguousarray(pad[idx]))
                    if peer == rank:
                        if kind == "send":
                            selfq.append(buf.clone())
                        else:
                            pad[idx] = selfq.pop(0).numpy()
                    elif kind == "send":
                        reqs.append((None, dist.isend(buf, peer)))
                    else:
                        reqs.append(((idx, buf), dist.irecv(buf, peer)))
                for meta, r in reqs:
                    r.wait()
                    if meta is not None:
                        idx, buf = meta
                        pad[idx] = buf.numpy()
            if bc == "fixed":
                s0 = 0 if has[(1, 0)] else h
                e0 = El[0] + 2 * h if has[(1, 1)] else El[0] + h
                s1 = 0 if has[(0, 0)] else h
                e1 = El[1] + 2 * h if has[(0, 1)] else El[1] + h
                res = oracle.run(np.ascontiguousarray(pad[s0:e0, s1:e1]), w, "fixed", step)
                local = res[h - s0:h - s0 + El[0], h - s1:h - s1 + El[1]]
            else:
                res = oracle.run(pad, w, "periodic", step)
                local = res[h:h + El[0], h:h + El[1]]
            done += step
        gathered = [None] * world if rank == 0 else None
        dist.gather_object((lo, hi, local), gathered, dst=0)
        if rank == 0:
            full = np.empty(ext)
            for blo, bhi, blk in gathered:
                full[tuple(slice(a, b) for a, b in zip(blo, bhi))] = blk
            ref = oracle.run(full0, w, bc, T)
            q.put(float(np.max(np.abs(full - ref)) / np.max(np.abs(ref))))
    except Exception as e:  # surface errors to the parent
        q.put(repr(e))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("p0,p1,bc,name,ext,T,tf", [
    (2, 2, "fixed", "box2d9p", (61, 40), 7, 3), (2, 2, "periodic", "box2d9p", (61, 40), 7, 3),
    (1, 2, "periodic", "box2d9p", (61, 40), 7, 3), (2, 2, "fixed", "heat3d", (14, 9, 10), 3, 1),
    (2, 2, "periodic", "heat3d", (14, 9, 10), 3, 1), (1, 2, "periodic", "box3d27p", (9, 12, 7), 2, 1),
    (2, 1, "fixed", "box3d27p", (9, 12, 7), 2, 1)])
def test_pencil_matches_single_domain(p0, p1, bc, name, ext, T, tf):
    """Pencil / block decomposition: corners and edges travel through the
    two-phase face exchange; the gathered blocks equal the single-domain oracle."""
    world = p0 * p1
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_pencil_worker, args=(r, world, port, p0, p1, name, ext, T, bc, tf, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
    assert not isinstance(res, str), res
    assert res <= 1e-13
