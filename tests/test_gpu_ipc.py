"""Multi-process peer path with real CUDA IPC: two processes (ranks of a G = 2 group) on
one B200, each with its own context and cache slab, exchanging cudaIpcMemHandles over a
gloo process group (ugache_ipc_handle / ugache_open_peers), sharing one /dev/shm host
table; each rank's extraction is compared byte for byte with the oracle."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, shm, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        import oracle
        import synth
        from oracle.placement import source_counts
        from paper_conf_sosp_songz0c23_b200 import UGache, dist as ugd
        torch.cuda.set_device(0)
        wl = synth.get_workload("tiny")
        if rank == 0:
            table = synth.HostTable(wl.num_rows, wl.row_bytes, shm_path=shm, create=True)
            table.fill()
        dist.barrier()
        if rank != 0:
            table = synth.HostTable(wl.num_rows, wl.row_bytes, shm_path=shm, create=False)
        h = synth.hotness(wl)
        cache = UGache(table, wl.num_rows, wl.row_bytes, wl.capacity_rows, hotness=h,
                       num_gpus=ws, rank=rank, device=0)
        ugd.connect(cache)
        cache.fill()
        torch.cuda.synchronize()
        ugd.barrier()                      # every slab filled before anyone reads a peer
        res = []
        for b in range(3):
            keys = synth.make_batch(wl, rank, b)
            out = cache.extract(torch.from_numpy(keys).cuda())
            torch.cuda.synchronize()
            ref, _ = oracle.gather(table.ptr, wl.num_rows, wl.row_bytes, keys)
            per, bad = cache.last_batch_stats()
            loc, _ = cache.export_placement()
            cnt, _ = source_counts(loc, keys, wl.num_rows, ws)
            res.append((bool(np.array_equal(out.cpu().numpy(), ref)),
                        bool(np.array_equal(per, cnt)), int(per[1 - rank])))
        ugd.barrier()                      # peers stay mapped until everyone is done
        cache.close()
        q.put((rank, res, None))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, None, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def test_two_process_ipc_peers_on_one_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    shm = f"/dev/shm/ugache_test_ipc_{os.getpid()}"
    ps = [ctx.Process(target=_worker, args=(r, 2, port, shm, q)) for r in range(2)]
    for p in ps:
        p.start()
    try:
        out = sorted(q.get(timeout=300) for _ in range(2))
    finally:
        for p in ps:
            p.join(timeout=60)
        if os.path.exists(shm):
            os.unlink(shm)
    for rank, res, err in out:
        assert err is None, err
        for same, counts_ok, n_peer in res:
            assert same and counts_ok
            assert n_peer > 0                 # rows really came from the other process's slab
