"""Per-select cost of the Python binding (wall time of enqueueing) vs the GPU time, and CUDA-graph
replay of K back-to-back selects (one graph launch; removes CPU enqueue cost and launch gaps).
    python tools/probe_graph.py [config ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

for cfg in sys.argv[1:] or ["c1", "c2"]:
    c = bench.CFG[cfg]
    x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
    k = c["k"]
    ws = torch.empty(at.workspace_bytes(x.dtype, c["batch"], c["n"], k), dtype=torch.uint8, device="cuda")
    ov = torch.empty((c["batch"], k), dtype=x.dtype, device="cuda")
    oi = torch.empty((c["batch"], k), dtype=torch.int64, device="cuda")
    steps = 200
    for _ in range(10):
        at.select(x, k, workspace=ws, out=(ov, oi))
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(steps):
        at.select(x, k, workspace=ws, out=(ov, oi))
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    # the C ABI call alone (ctypes, prebuilt arguments): library host cost + launch API
    import ctypes
    L = at.lib()
    o = at._opts()
    args = (x.data_ptr(), at.dtype_code(x.dtype), c["batch"], c["n"], k, 1, ov.data_ptr(), oi.data_ptr(),
            ws.data_ptr(), ws.numel(), torch.cuda.current_stream().cuda_stream, ctypes.byref(o))
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    for _ in range(steps):
        L.airtopk_select_ex(*args)
    t4 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"{cfg}: C ABI call alone {(t4 - t3) / steps * 1e6:.1f} us/select", flush=True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        at.select(x, k, workspace=ws, out=(ov, oi))
    e1.record()
    torch.cuda.synchronize()
    eager = e0.elapsed_time(e1) / steps * 1e3
    # graph of `per` selects, replayed
    per = 20
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    try:
        with torch.cuda.stream(s):
            at.select(x, k, workspace=ws, out=(ov, oi))
            torch.cuda.current_stream().synchronize()
            with torch.cuda.graph(g, stream=s):
                for _ in range(per):
                    at.select(x, k, workspace=ws, out=(ov, oi))
        torch.cuda.synchronize()
        for _ in range(3):
            g.replay()
        torch.cuda.synchronize()
        e0.record()
        for _ in range(steps // per):
            g.replay()
        e1.record()
        torch.cuda.synchronize()
        graph = e0.elapsed_time(e1) / (steps // per * per) * 1e3
        rv, ri = at.select(x, k)
        ok = torch.equal(torch.sort(ri, dim=1).values, torch.sort(oi, dim=1).values)
    except Exception as e:  # noqa: BLE001
        graph, ok = float("nan"), repr(e)[:200]
    print(f"{cfg}: python enqueue {(t1 - t0) / steps * 1e6:.1f} us/select (wall to drain {(t2 - t0) / steps * 1e6:.1f}); "
          f"eager GPU {eager:.1f} us/select; graph replay {graph:.1f} us/select; graph result ok: {ok}", flush=True)
