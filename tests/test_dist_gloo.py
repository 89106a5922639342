"""Multi-process (world_size 2 and 3, gloo, CPU) tests of the multi-GPU partition / gather / merge
logic of paper_conf_sc_zhangnlw23_b200.dist. The local selects are the CPU oracle here (tests may
use it); on GPUs the same code calls the CUDA kernels. Checks the SURVEY §8(e) argument: the
merged top-K of per-shard top-Ks equals the single-row top-K, including ties across shards."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_shard(t, k, off, pad_base, largest, out):
    """The contract of airtopk_select_shard, on the CPU oracle: the shard's top min(k, n) with
    global indices, then pads (keys that sort last, indices pad_base + j)."""
    from paper_conf_sc_zhangnlw23_b200 import dist as atd
    x = t.numpy().reshape(1, -1)
    kk = min(k, x.shape[1])
    v, i = oracle.topk_sort(x, kk, select_min=not largest)
    ov, oi = out
    ov[:kk] = torch.from_numpy(v[0])
    oi[:kk] = torch.from_numpy(i[0]) + off
    if kk < k:
        bits = atd.pad_bits(t.dtype, largest)
        ov[kk:] = torch.from_numpy(np.full(k - kk, bits, dtype=np.uint32).view(np.float32))
        oi[kk:] = pad_base + torch.arange(k - kk)


def _oracle_merge(gv, gi, k, idx_bits, largest):
    assert int(gi.max()) < (1 << idx_bits)
    v, i = oracle.topk_with_idx(gv.numpy(), gi.numpy(), k, select_min=not largest)
    return torch.from_numpy(v), torch.from_numpy(i)


def _one(rank, world, case):
    from paper_conf_sc_zhangnlw23_b200 import dist as atd
    if case["kind"] == "split":
        n_total, k, largest = case["n"], case["k"], case["largest"]
        bounds = np.linspace(0, n_total, world + 1).astype(np.int64)
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        x = gen.keys(case["dist"], 7, n_total, m_bits=case.get("m", 20))
        v, i = atd.select_split_row(torch.from_numpy(x[lo:hi].copy()), k, total_len=n_total, shard_offset=lo,
                                    largest=largest, shard_fn=_oracle_shard, merge_fn=_oracle_merge)
        rv, ri = oracle.topk_sort(x, k, select_min=not largest)
        ok = np.array_equal(np.sort(i.numpy()), np.sort(ri[0]))
        ok &= np.array_equal(np.sort(v.numpy().view(np.uint32)), np.sort(rv[0].view(np.uint32)))
        return bool(ok)
    batch, n, k = case["batch"], case["n"], case["k"]
    lo, hi = atd.row_range(batch, rank, world)
    x = gen.keys("normal", 3, batch * n).reshape(batch, n)
    v, i, _ = atd.select_rows(torch.from_numpy(x[lo:hi].copy()), k,
                              select_fn=lambda t, kk, lg: tuple(torch.from_numpy(a) for a in
                                                                oracle.topk_nth(t.numpy(), kk, not lg)))
    rv, ri = oracle.topk_nth(x[lo:hi], k)
    ok = np.array_equal(i.numpy(), ri)
    sizes = [None] * world
    dist.all_gather_object(sizes, hi - lo)
    return bool(ok and sum(sizes) == batch)


def _worker(rank, world, port, cases, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, [_one(rank, world, c) for c in cases]))
    finally:
        dist.destroy_process_group()


def _run(world, cases):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, cases, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, oks in res:
        bad = [c for c, ok in zip(cases, oks) if not ok]
        assert not bad, f"rank {rank} failed: {bad}"


SPLIT_CASES = [dict(kind="split", n=30011, k=700, dist=d, m=m, largest=lg)
               for d, m in (("uniform", 20), ("adversarial", 28), ("adversarial", 31)) for lg in (False, True)]


@pytest.mark.parametrize("world", [2, 3])
def test_split_row_merge_and_row_sharding(world):
    cases = SPLIT_CASES + [dict(kind="rows", batch=10, n=5000, k=37)]
    if world == 3:
        # every shard shorter than K: padding candidates must never be selected
        cases.append(dict(kind="split", n=1000, k=600, dist="adversarial", m=30, largest=False))
        cases.append(dict(kind="split", n=1000, k=600, dist="uniform", m=20, largest=True))
    _run(world, cases)


def test_row_range_partition():
    from paper_conf_sc_zhangnlw23_b200 import dist as atd
    for batch in (1, 7, 100):
        for world in (1, 2, 4, 8):
            rr = [atd.row_range(batch, r, world) for r in range(world)]
            assert rr[0][0] == 0 and rr[-1][1] == batch
            assert all(rr[i][1] == rr[i + 1][0] for i in range(world - 1))
            sizes = [b - a for a, b in rr]
            assert max(sizes) - min(sizes) <= 1


def test_pad_bits_sort_last():
    from paper_conf_sc_zhangnlw23_b200 import dist as atd
    for dt, dtn, npdt in ((torch.float32, "f32", np.uint32), (torch.float16, "f16", np.uint16),
                          (torch.float64, "f64", np.uint64), (torch.uint32, "u32", np.uint32)):
        for largest in (False, True):
            b = atd.pad_bits(dt, largest)
            c = oracle.codes(np.array([b], npdt), select_min=not largest, dt=oracle.DT_NAMES[dtn])[0]
            assert int(c) == (1 << oracle.rbits(oracle.DT_NAMES[dtn])) - 1
