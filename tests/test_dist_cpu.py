"""Control plane over torch.distributed with the gloo backend, world size 2, on CPU:
IPC-handle exchange with the placement digest, max/sum over ranks, per-rank row gather."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, q, same_digest):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    from paper_conf_sosp_songz0c23_b200 import dist as ugd
    try:
        digest = ugd.placement_digest({"k": 5, "band_end": 9}, np.arange(10, dtype=np.uint64))
        if not same_digest and rank == 1:
            digest = ugd.placement_digest({"k": 6, "band_end": 9}, None)
        handles = ugd.exchange_handles(bytes([rank]) * 64, digest)
        mx = ugd.max_over_ranks(float(rank + 1))
        sm = ugd.sum_over_ranks(float(rank + 1))
        rows = ugd.gather_rows([rank, 10.0 * rank + 1, -rank])
        ugd.barrier()
        q.put((rank, [h[0] for h in handles], mx, sm, rows.tolist(), None))
    except Exception as e:  # noqa: BLE001
        q.put((rank, None, None, None, None, repr(e)))
    finally:
        dist.destroy_process_group()


def _run(same_digest):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q, same_digest)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in ps:
        p.join(timeout=60)
    return sorted(res)


def test_handle_exchange_and_reductions_gloo_ws2():
    res = _run(True)
    for rank, handles, mx, sm, rows, err in res:
        assert err is None, err
        assert handles == [0, 1]          # rank order
        assert mx == 2.0 and sm == 3.0
        assert rows == [[0.0, 1.0, 0.0], [1.0, 11.0, -1.0]]   # every rank's row, rank order


def test_placement_digest_mismatch_is_detected():
    res = _run(False)
    assert all(err is not None and "different placements" in err for _, _, _, _, _, err in res)
