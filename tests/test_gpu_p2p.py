"""NEXT #2 (collective-fused exchange over peer memory, csrc/p2p.cu): two processes on ONE GPU
(CUDA IPC works between processes on the same device; over NVLink the same stores are P2P writes),
handles exchanged over gloo. The split-row select through PeerExchange must equal the oracle's
single-row top-K, repeatedly (epochs), including shards shorter than K. Unmeasured on NVLink here."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

CASES = [(3 << 18, 5000, "uniform", False), (300_001, 4096, "adversarial", False), (3000, 2000, "normal", True)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import gen
        from paper_conf_sc_zhangnlw23_b200 import dist as atd
        torch.cuda.set_device(0)
        results = []
        for n, k, distn, largest in CASES:
            x = gen.keys(distn, 61, n, m_bits=26)
            bounds = np.linspace(0, n, world + 1).astype(np.int64)
            lo, hi = int(bounds[rank]), int(bounds[rank + 1])
            ex = atd.PeerExchange(k, torch.float32, torch.device("cuda", 0))
            xs = torch.from_numpy(x[lo:hi].copy()).cuda()
            for _ in range(3):  # epochs
                v, i = atd.select_split_row_p2p(xs, k, n, lo, ex, largest=largest)
                torch.cuda.synchronize()
            results.append((v.cpu().numpy(), i.cpu().numpy()))
            dist.barrier()
            ex.close()
        q.put((rank, results))
    finally:
        dist.destroy_process_group()


def test_peer_exchange_split_row_two_processes():
    import torch.multiprocessing as mp
    import gen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world = 2
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=240) for _ in ps)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for ci, (n, k, distn, largest) in enumerate(CASES):
        x = gen.keys(distn, 61, n, m_bits=26)
        rv, ri = oracle.topk_sort(x, k, select_min=not largest)
        for r in range(world):
            v, i = res[r][ci]
            assert np.array_equal(np.sort(i), np.sort(ri[0])), (ci, r)
            assert np.array_equal(np.sort(v.view(np.uint32)), np.sort(rv[0].view(np.uint32)))
