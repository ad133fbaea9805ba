"""Multi-process peer path with real CUDA IPC: two processes (ranks of a G = 2 group) on
one B200, each with its own context and cache slab, exchanging cudaIpcMemHandles over a
gloo process group (ugache_ipc_handle / ugache_open_peers), sharing one /dev/shm host
table; each rank's extraction is compared byte for byte with the oracle -- factored
extraction, the message-based baseline over the process group, and a chunked cache
refresh driven across the two processes."""
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
        # the message-based baseline over the real process group (all-to-alls staged through
        # host memory on gloo), same batch, same placement
        from paper_conf_sosp_songz0c23_b200.message import message_extract
        keys = synth.make_batch(wl, rank, 0)
        out = message_extract(cache, torch.from_numpy(keys).cuda())
        torch.cuda.synchronize()
        ref, _ = oracle.gather(table.ptr, wl.num_rows, wl.row_bytes, keys)
        msg_ok = bool(np.array_equal(out.cpu().numpy(), ref))
        # chunked refresh across the two processes (barriers between the steps), to a
        # placement solved for a permuted hotness; extraction stays bit-exact throughout
        from paper_conf_sosp_songz0c23_b200.refresh import plan_placements, refresh_distributed
        h2 = h[np.random.default_rng(5).permutation(len(h))]
        _, pl2 = plan_placements(dict(num_rows=wl.num_rows, row_bytes=wl.row_bytes,
                                      capacity_rows=wl.capacity_rows), h2, ws)
        fg_ok = []

        def foreground():
            k2 = synth.make_batch(wl, rank, 7)
            o2 = cache.extract(torch.from_numpy(k2).cuda())
            torch.cuda.synchronize()
            r2, _ = oracle.gather(table.ptr, wl.num_rows, wl.row_bytes, k2)
            fg_ok.append(bool(np.array_equal(o2.cpu().numpy(), r2)))

        refresh_distributed(cache, pl2[rank], max_sms=4, max_rows=3000, foreground=foreground)
        foreground()
        loc2, sk2 = cache.export_placement()
        refreshed = bool(np.array_equal(loc2, pl2[rank][0]) and np.array_equal(sk2, pl2[rank][1]))
        res.append((msg_ok and all(fg_ok) and len(fg_ok) >= 3 and refreshed, True, 1))
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
