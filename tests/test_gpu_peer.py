"""GPU parity of the NVLink peer-memory halo exchange (csx_run_sharded_peer).

Two checks, both against the single-domain CPU oracle (max rel. error <= 1e-12):
  * one rank on a PERIODIC ring (the rank is its own up / down neighbour: the push kernel copies
    the slab's boundary rows into its own ghost rows and publishes the epochs to itself), with
    and without the overlapped interior / edge schedule, over several back-to-back runs (epochs
    carry across runs);
  * two processes sharing cuda:0 (gloo bootstrap, CUDA IPC mappings of each other's slab
    buffers and flag blocks — the same code path as one process per GPU over NVLink), FIXED and
    PERIODIC, 1D / 2D / 3D.  The slabs are gathered and compared with the oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

TOL = 1e-12


def rel(a, b):
    return float(np.max(np.abs(a - b)) / np.max(np.abs(b)))


@pytest.fixture(scope="module")
def csx():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ppopp_chenlwbwmyzcy24_b200 as m
    return m


@pytest.mark.parametrize("overlap", ["0", "1"])
@pytest.mark.parametrize("name,ext,T", [("box2d9p", (200, 130), 10), ("heat1d", (30000,), 23),
                                        ("box3d27p", (40, 30, 40), 4), ("star2d13p", (150, 90), 3)])
def test_peer_single_rank_ring(csx, monkeypatch, overlap, name, ext, T):
    monkeypatch.setenv("CSX_FORCE_OVERLAP", overlap)
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=21)
    p = csx.Plan(u0.shape, w, shape=s.kind, bc="periodic")
    p.peer_setup(0, 1)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    ref = oracle.run(u0, w, "periodic", T)
    for _ in range(3):  # epochs continue across runs
        p.run_sharded_peer(d_in, d_out, T, u0.size)
        torch.cuda.synchronize()
        assert rel(d_out.cpu().numpy(), ref) <= TOL, (name, overlap)
    p.close()


def test_peer_api_errors(csx):
    w = synth.physical_weights("box2d9p")
    p = csx.Plan((64, 64), w, bc="fixed")
    d = torch.zeros(64 * 64, dtype=torch.float64, device="cuda")
    with pytest.raises(csx.CsxError):  # not exported / connected
        p.run_sharded_peer(d, d, 3, d.numel())
    with pytest.raises(csx.CsxError):
        csx.csx_peer_connect(p.handle, [b"\0" * csx.CSX_PEER_DESC_BYTES])
    desc = csx.csx_peer_export(p.handle, 0, 1)
    with pytest.raises(csx.CsxError):  # exported twice
        csx.csx_peer_export(p.handle, 0, 1)
    bad = bytearray(desc)
    bad[0] ^= 0xFF
    with pytest.raises(csx.CsxError):  # corrupted descriptor
        csx.csx_peer_connect(p.handle, [bytes(bad)])
    csx.csx_peer_connect(p.handle, [desc])
    p.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, cases, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
        torch.cuda.set_device(0)
        res = []
        for name, ext, T, bc in cases:
            s = synth.SHAPES[name]
            w = synth.random_weights(name)
            p = csx.Plan(ext, w, shape=s.kind, bc=bc)
            p.peer_setup(rank, world)
            lo, hi = p.shard_rows(rank, world)
            u0 = synth.grid(ext, rows=(lo, hi), seed=33)
            d_in = torch.from_numpy(np.ascontiguousarray(u0)).cuda()
            d_out = torch.empty_like(d_in)
            for _ in range(2):
                p.run_sharded_peer(d_in, d_out, T, u0.size)
            torch.cuda.synchronize()
            res.append((lo, hi, d_out.cpu().numpy()))
            dist.barrier()
            p.close()
        q.put((rank, res, None))
    except Exception as e:  # report to the parent
        q.put((rank, None, repr(e)))
    finally:
        dist.destroy_process_group()


CASES = [("box2d9p", (160, 130), 10, "fixed"), ("box2d9p", (161, 130), 7, "periodic"),
         ("heat1d", (20001,), 23, "fixed"), ("heat1d", (20000,), 12, "periodic"),
         ("box3d27p", (30, 24, 40), 4, "periodic"), ("heat3d", (31, 24, 40), 3, "fixed")]


def test_peer_two_processes_one_gpu(csx):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    world = 2
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, CASES, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = {}
    for _ in range(world):
        rank, res, err = q.get(timeout=600)
        assert err is None, f"rank {rank}: {err}"
        out[rank] = res
    for pr in procs:
        pr.join(timeout=60)
    for k, (name, ext, T, bc) in enumerate(CASES):
        w = synth.random_weights(name)
        u0 = synth.grid(ext, seed=33)
        got = np.concatenate([out[r][k][2] for r in range(world)], axis=0)
        assert got.shape == u0.shape
        assert rel(got, oracle.run(u0, w, bc, T)) <= TOL, (name, ext, bc)
