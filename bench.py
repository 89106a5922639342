#!/usr/bin/env python
"""bench.py — AIR Top-K on B200: top-K elements/s and achieved HBM GB/s vs B200 peak.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl ours|reference]

One "step" = one full AIR Top-K select (every radix pass + the last filter) over the
config's synthetic input, already resident in HBM. Default workload = c3 (batch 1, N = 2^30
uniform (0,1] f32, K = 2^20, select-min), the configuration BASELINE.json's metric is quoted on.

N > 1 (torchrun, one rank per GPU, NCCL):
  c3/c5-style: one row of N * 2^30 elements split across the ranks (per-GPU work fixed -> "weak"):
      local select of the 2^30 shard + NCCL all-gather of the K candidates + merge select.
  c2: the 100 rows are sharded across ranks (total work fixed -> "strong"), no collective.

The oracle (oracle/, CPU) is executed ONLY by the cpu_baseline leg and by --impl reference.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402

PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM_GBS = 6650.0  # /opt/skills/guides/B200_PROFILING.md fallback

CFG = {
    "c1": dict(batch=1, n=1 << 16, k=32, dist="uniform"),
    "c2": dict(batch=100, n=1 << 20, k=256, dist="normal"),
    "c3": dict(batch=1, n=1 << 30, k=1 << 20, dist="uniform"),
    "c4": dict(batch=1, n=1 << 28, k=50000, dist="adversarial"),
    # one 2^33 row: on one GPU the whole row (64-bit index path), at N ranks a 2^33/N shard each
    "c5": dict(batch=1, n=1 << 33, k=1 << 16, dist="uniform"),
}
DEFAULT_STEPS = {"c1": 500, "c2": 300, "c3": 200, "c4": 200, "c5": 10}  # timed regions >= ~0.1 s (clock samples)


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def hbm_peak():
    try:
        with open(PEAKS_FILE) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback"


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi sampling of SM clocks and throttle reasons during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        time.sleep(0.12)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- inputs
def host_keys(cfg_name: str, n: int, batch: int, offset: int = 0):
    c = CFG[cfg_name]
    seed = gen.config_seed(cfg_name)
    return gen.keys(c["dist"], seed, batch * n, offset=offset).reshape(batch, n)


def n_passes(n: int, R: int = 32):
    ib = int(n - 1).bit_length()
    return -(-R // 11) + -(-ib // 11)


# ----------------------------------------------------------------------------- reference arm / CPU baseline
METRIC = "top-K elements/s and achieved HBM GB/s vs B200 peak (N=2^30,K=2^20; b=100)"


def cpu_info():
    """lscpu model name, usable cores and OMP_NUM_THREADS of this host."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.lower().startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    try:
        usable = len(os.sched_getaffinity(0))
    except Exception:
        usable = os.cpu_count()
    return {"lscpu_model": model, "nproc": usable, "cpu_count": os.cpu_count(),
            "OMP_NUM_THREADS": os.environ.get("OMP_NUM_THREADS")}


def _time_oracle(fn, budget_s, min_reps=1):
    reps, t0 = 0, time.perf_counter()
    while True:
        r = fn()
        reps += 1
        el = time.perf_counter() - t0
        if reps >= min_reps and el >= budget_s:
            return reps, el, r


def cpu_sample_run(cfg_name: str, budget_s: float):
    """Time the CPU oracle as it stands on a bounded sample of the workload (same distribution and
    K/N ratio, N_s = min(N, 2^26) per row): the all-cores variant (oracle.topk_nth_mt, OpenMP) is
    the reported value; the single-core oracle.topk_nth is timed beside it."""
    import oracle
    c = CFG[cfg_name]
    ns = min(c["n"], 1 << 26)
    ks = max(1, round(c["k"] * ns / c["n"]))
    rows = 1 if c["batch"] == 1 else min(c["batch"], max(1, (1 << 26) // ns))
    x = host_keys(cfg_name, ns, rows)
    oracle.build()
    oracle.topk_nth(x[:1, : min(ns, 1 << 16)], min(ks, 1 << 16))  # load / warm
    reps, el, r = _time_oracle(lambda: oracle.topk_nth_mt(x, ks), budget_s / 2)
    threads = r[2]
    reps1, el1, _ = _time_oracle(lambda: oracle.topk_nth(x, ks), budget_s / 2)
    info = cpu_info()
    return {"value": reps * rows * ns / el, "unit": "elements/s", "cores": threads, "kind": "oracle",
            "variant": "oracle.topk_nth_mt (OpenMP chunks + candidate merge, all cores)",
            "single_core": {"value": reps1 * rows * ns / el1, "cores": 1, "variant": "oracle.topk_nth",
                            "reps": reps1, "seconds": el1},
            "sample": f"{reps} x oracle.topk_nth_mt on {rows} x 2^{int(math.log2(ns))} {c['dist']} f32, K={ks} "
                      f"(same K/N as {cfg_name}), {el:.1f} s on {threads} threads",
            **info}


def run_reference(args, rank):
    """The reference arm: this tier's reference is the CPU oracle (the paper ships no code). It runs
    the repo arm's exact metric and workload (the real config input, e.g. c3 = 2^30 keys) on the
    host cores: one untimed warm-up select, then as many timed selects as fit in --ref-budget
    seconds (at least one); `steps` = the selects actually timed."""
    if rank != 0:
        return
    import oracle
    cfg = args.config
    c = CFG[cfg]
    oracle.build()
    t0 = time.perf_counter()
    x = host_keys(cfg, c["n"], c["batch"])
    gen_s = time.perf_counter() - t0
    oracle.topk_nth_mt(x, c["k"])  # warm-up (allocation, page faults)
    reps, el, r = _time_oracle(lambda: oracle.topk_nth_mt(x, c["k"]), args.ref_budget)
    threads = r[2]
    value = reps * c["batch"] * c["n"] / el
    cb = {"value": value, "unit": "elements/s", "cores": threads, "kind": "oracle",
          "variant": "oracle.topk_nth_mt (OpenMP chunks + candidate merge, all cores)",
          "sample": f"the full {cfg} input ({c['batch']} x {c['n']} {c['dist']} f32, K={c['k']}): "
                    f"{reps} timed selects in {el:.1f} s after 1 warm-up (input generated in {gen_s:.1f} s)",
          **cpu_info()}
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "elements/s",
            "n_gpus": args.gpus, "steps": reps, "warmup": 1, "steps_requested": args.steps,
            "ms_per_step": el / reps * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": cfg, "batch": c["batch"], "n": c["n"], "k": c["k"], "dist": c["dist"]},
            "cpu_baseline": cb, "e2e": {"value": value, "unit": "elements/s", "h2d_bytes_per_step": 0,
                                        "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def maybe_relaunch(args):
    """`bench.py --gpus N` (N > 1) outside torchrun: re-exec under torch.distributed.run with N
    ranks on this node (the driver's own launch sets WORLD_SIZE, so it runs directly)."""
    if args.gpus <= 1 or "WORLD_SIZE" in os.environ or args.impl == "reference":
        return
    import socket
    so = socket.socket()
    so.bind(("127.0.0.1", 0))
    port = so.getsockname()[1]
    so.close()
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")          # communicator lines show nranks / NVLS
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    log("relaunching under torchrun:", " ".join(cmd))
    os.execve(sys.executable, cmd, env)


# ----------------------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=None)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="c3", choices=sorted(CFG))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-extras", action="store_true", help="skip the c1/c2/c4 side measurements")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--cpu-budget", type=float, default=10.0)
    ap.add_argument("--ref-budget", type=float, default=30.0)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--engine", type=int, default=0, help="0 auto, 1 grid, 2 cluster (ablations)")
    ap.add_argument("--dtype", default="f32", choices=["f32", "f16", "bf16", "f64", "u32"],
                    help="key type (f32: the paper's; others: the config's f32 keys converted)")
    ap.add_argument("--window", type=int, default=0, help="sample-guided window: 0 auto, 1 on, -1 off (ablation)")
    ap.add_argument("--tma", type=int, default=0, help="bulk-copy streaming: 0 auto, 1 on, -1 off (ablation)")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "p2p"],
                    help="split-row candidate exchange: one NCCL all-gather, or peer stores over CUDA IPC "
                         "(PeerExchange, SURVEY §8(f) NEXT #2)")
    ap.add_argument("--dist-backend", default="nccl", help="nccl (default); gloo only to self-test the "
                    "multi-rank flow with several ranks on one GPU")
    args = ap.parse_args()
    if args.steps is None:
        args.steps = DEFAULT_STEPS[args.config]
    args.warmup = max(3, args.warmup)
    maybe_relaunch(args)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_sc_zhangnlw23_b200 as at
    from paper_conf_sc_zhangnlw23_b200 import dist as atdist

    ndev = torch.cuda.device_count()
    local_dev = local % max(1, ndev)  # (> 1 rank per GPU only for the --dist-backend gloo self-test)
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(args.dist_backend)
    at.lib()

    cfg = args.config
    c = CFG[cfg]
    peak, peak_kind = hbm_peak()

    # ---------------- workload on this rank
    if cfg == "c5":  # the fixed 2^33 row split across the ranks (total work fixed -> "strong")
        batch, n = 1, c["n"] // world
        xh = host_keys(cfg, n, 1, offset=rank * n)
        scaling = "strong"
        total_units = c["n"]
        split = world > 1
    elif cfg == "c2":
        lo, hi = atdist.row_range(c["batch"], rank, world)
        batch, n = hi - lo, c["n"]
        xh = host_keys(cfg, n, batch, offset=lo * n)
        scaling = "strong"
        total_units = c["batch"] * c["n"]
        split = False
    else:
        batch, n = c["batch"], c["n"]
        xh = host_keys(cfg, n, batch, offset=rank * n * batch)
        scaling = "weak"
        total_units = world * batch * n
        split = world > 1
    k = c["k"]
    xt = keys_as(torch.from_numpy(xh), args.dtype)
    kdt = xt.dtype
    esz = xt.element_size()
    xd = xt.to(dev)
    sel_opts = dict(engine=args.engine, window=args.window, tma=args.tma)
    ws = torch.empty(max(1, at.describe(kdt, batch, n, k, **sel_opts)["workspace_bytes"]),
                     dtype=torch.uint8, device=dev)
    ov = torch.empty((batch, k), dtype=kdt, device=dev)
    oi = torch.empty((batch, k), dtype=torch.int64, device=dev)
    plan = at.describe(kdt, batch, n, k, **sel_opts)
    n_launch = plan["launches"]
    stream = torch.cuda.current_stream(dev)
    ev_sets = []

    total_len = (c["n"] if cfg == "c5" else world * n)
    if split:  # gather buffers reused every step; the shard select writes into slot `rank` in place
        gbuf = (torch.empty(world * k, dtype=kdt, device=dev), torch.empty(world * k, dtype=torch.int64, device=dev))
        ws_shard = torch.empty(max(1, at.lib().airtopk_workspace_bytes_shard(at.dtype_code(kdt), n, k)),
                               dtype=torch.uint8, device=dev)
        mbits = at.merge_idx_bits(total_len, world, k)
        ws_merge = torch.empty(max(1, at.lib().airtopk_workspace_bytes_with_idx(at.dtype_code(kdt), world * k, k,
                                                                                  mbits)), dtype=torch.uint8, device=dev)
        mout = (torch.empty(k, dtype=kdt, device=dev), torch.empty(k, dtype=torch.int64, device=dev))

    if split and args.exchange == "p2p":
        pex = atdist.PeerExchange(k, kdt, dev)

    def step(events=None):
        if split and args.exchange == "p2p":
            return atdist.select_split_row_p2p(xd.reshape(-1), k, total_len, rank * n, pex, workspace=ws_shard,
                                               merge_workspace=ws_merge, out=mout)
        if split:
            return atdist.select_split_row(
                xd.reshape(-1), k, total_len=total_len, shard_offset=rank * n, buffers=gbuf,
                shard_fn=lambda t, kk, off, pb, lg, out: at.select_shard(t, kk, off, pb, largest=lg, out=out,
                                                                         workspace=ws_shard),
                merge_fn=lambda a, b, kq, ib, lg: at.select_with_idx(a, b, kq, ib, largest=lg, workspace=ws_merge,
                                                                     out=mout))
        return at.select(xd, k, workspace=ws, out=(ov, oi), events=events, **sel_opts)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # per-kernel events for every timed step (recorded on the launching stream by the library)
    for _ in range(args.steps):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(n_launch + 1)]
        for e in evs:
            e.record(stream)  # creates the cudaEvent_t; the library re-records it between launches
        ev_sets.append((evs, at.make_event_array(evs)))
    torch.cuda.synchronize()

    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.15)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for s_i in range(args.steps):
        step()
    t_end.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    # breakdown: the same K local selects again with the library recording a CUDA event between its
    # launches (events between launches defeat programmatic dependent launch, so the headline is
    # taken above; for a split row this times the shard's local select only)
    for s_i in range(args.steps):
        at.select(xd, k, workspace=ws, out=(ov, oi), events=ev_sets[s_i][1], **sel_opts)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    ms_local = t_start.elapsed_time(t_end) / args.steps
    ms = ms_local
    if world > 1:
        tt = torch.tensor([ms_local], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())

    # per-kernel durations (the select's launches; the merge path for N>1 is not in these events)
    per = np.zeros(n_launch)
    for evs, _ in ev_sets:
        for q in range(n_launch):
            per[q] += evs[q].elapsed_time(evs[q + 1])
    per /= args.steps
    select_ms = float(per.sum())
    dom = int(np.argmax(per))
    in_bytes = batch * n * esz
    out_bytes = batch * k * (esz + 8)
    # algorithmic bytes of the dominant kernel: passes that read the input read N*4 bytes once
    # (grid engine: launch 0 and 1 read L; cluster engine: its single launch reads the rows)
    names, reads_L = launch_names(plan)
    dom_alg = in_bytes if reads_L[dom] else None
    value = total_units / (ms * 1e-3)

    # ---------------- correctness spot check of the timed configuration (sampled, no oracle):
    v_chk, i_chk = step()
    torch.cuda.synchronize()

    result = None
    if rank == 0:
        roofline = None
        if dom_alg is not None:
            ach = dom_alg / (per[dom] * 1e-3) / 1e9
            roofline = {"bound": "hbm", "kernel": names[dom], "achieved": ach, "peak": peak,
                        "peak_kind": peak_kind, "unit": "GB/s", "frac": ach / peak,
                        "peak_note": "MEASURED_PEAKS hbm_gbs is a copy (read+write) rate; a read-only "
                                     "stream can exceed it (frac slightly > 1)",
                        "traffic": load_traffic(plan_key(cfg, plan, sel_opts, args.dtype), dom),
                        "traffic_plan": plan_key(cfg, plan, sel_opts, args.dtype),
                        "alg_bytes_per_launch": dom_alg, "launch_ms": float(per[dom])}
        whole = (in_bytes + out_bytes) / (select_ms * 1e-3) / 1e9
        result = {
            "metric": METRIC,
            "value": value, "unit": "elements/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms, "higher_is_better": True, "scaling": scaling, "vs_baseline": None,
            "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": cfg, "batch": c["batch"], "n": n, "k": k, "dist": c["dist"], "select": "min",
                       "per_gpu_rows": batch, "split_row": split,
                       "exchange": (args.exchange if split else None),
                       "l2": "input (%.2f GB) larger than L2 (126 MB): no flush needed" % (in_bytes / 1e9)
                       if in_bytes > (256 << 20) else "input smaller than L2: consecutive steps may hit L2",
                       "parallelism": f"{'split-row' if split else ('rows' if cfg == 'c2' else 'replica')}x{world}"},
            "roofline": roofline,
            "whole_select": {"achieved_gbs": whole, "frac": whole / peak, "ms": select_ms,
                             "alg_bytes": in_bytes + out_bytes,
                             "per_kernel_ms": [float(x) for x in per]},
            "gpu_launches": args.steps * (n_launch + (plan_merge_launches(world, k) if split else 0)),
            "plan": plan,
            "clocks": clocks,
        }
    # ---------------- e2e through the C ABI with HOST buffers (pinned), N GPUs, same metric
    xpin = xt.pin_memory()
    ovh = torch.empty((batch, k), dtype=kdt).pin_memory()
    oih = torch.empty((batch, k), dtype=torch.int64).pin_memory()
    at.select_host(xpin, k, out=(ovh, oih))
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(args.e2e_steps):
        at.select_host(xpin, k, out=(ovh, oih))
    el = (time.perf_counter() - t0) / args.e2e_steps
    if world > 1:
        tt = torch.tensor([el], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        el = float(tt.item())
    if rank == 0:
        result["e2e"] = {"value": total_units / el, "unit": "elements/s", "ms_per_step": el * 1e3,
                         "h2d_bytes_per_step": in_bytes, "d2h_bytes_per_step": out_bytes,
                         "path": "airtopk_select_host (pinned H2D + select + D2H + stream sync)"
                                 + (" of each rank's shard; the candidate all-gather + merge are not in e2e"
                                    if split else "")}
    del xpin

    if rank == 0:
        # oracle-free sanity of the timed output: K distinct indices, values = keys[idx]
        ii = i_chk.reshape(-1)[: min(k, 4096)].cpu().numpy()
        if not split:
            xb = xt.reshape(-1).view({1: torch.uint8, 2: torch.int16, 4: torch.int32, 8: torch.int64}[esz])
            vb = v_chk.reshape(-1)[: min(k, 4096)].view(xb.dtype).cpu()
            assert torch.equal(xb[torch.from_numpy(ii)], vb), "value/index mismatch"
        if not args.no_cpu:
            result["cpu_baseline"] = cpu_sample_run(cfg, args.cpu_budget)
        if world == 1 and not args.no_extras and cfg == "c3":
            del xd, ws, ov, oi
            torch.cuda.empty_cache()
            result["extras"] = {name: extra_measure(name, dev) for name in ("c1", "c2", "c4")}
            result["per_rank_proxies"] = per_rank_proxies(dev)
        print(json.dumps(result), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def keys_as(xt, dtype):
    """The config's f32 keys as another key type (f16/bf16/f64 by value conversion, u32 by the
    order-preserving bit pattern of the positive f32 values)."""
    import torch
    if dtype == "f32":
        return xt
    if dtype == "f16":
        return xt.half()
    if dtype == "bf16":
        return xt.bfloat16()
    if dtype == "f64":
        return xt.double()
    return xt.view(torch.int32).view(torch.uint32)


def launch_names(plan):
    """Names of a select's launches in order, and whether each streams the input row L once (its
    algorithmic bytes are then N*4; SURVEY §8(d) per-element figure x elements per launch)."""
    if plan["engine"] == 2:
        return ["cluster_kernel (all passes)"], [True]
    if plan["engine"] == 3:
        return ["trivial_copy"], [True]
    if plan["engine"] == 4:
        return ["gridselect_kernel (GridSelect, P:188-204)"], [True]
    if plan["engine"] == 5:
        return ["batch_kernel (sample + window stream + finish)", "cluster_kernel (fallback rows)"], [True, False]
    P = plan["passes"]
    L = plan["launches"]
    if plan["engine"] == 1 and L in (1, 3):  # fused tail: [sample, window pass,] one launch for the rest
        if L == 1:
            return ["tail_kernel (all passes, from L)"], [True]
        return ["sample_kernel", "window_pass (DF=3)", "tail_kernel (remaining passes)"], [False, True, False]
    if L not in (P + 1, P + 3):  # window pass + tail_q grid passes + one cluster-engine tail launch
        tq = L - 3
        names = ["sample_kernel", "window_pass (DF=3)"] + [f"pass_kernel q={q} [window buffer]" for q in range(tq)]
        names.append("cluster_kernel (tail)")
        return names, [False, True] + [False] * (tq + 1)
    window = L == P + 3
    names, reads = [], []
    if window:
        names += ["sample_kernel", "window_pass (DF=3)"]
        reads += [False, True]
    for q in range(P + 1):
        nm = "last_filter (q=P)" if q == P else f"pass_kernel q={q}"
        names.append(nm + (" [window buffer]" if window and q <= 1 else ""))
        reads.append((not window) and q <= 1)
    return names, reads


def plan_merge_launches(world, k):
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    return at.describe(torch.float32, 1, world * k, k)["launches"]


def plan_key(cfg, plan, sel_opts, dtype="f32"):
    """Identifies a launch sequence: config, key type, engine, launch count and the window / bulk-copy
    options (the same config runs different kernels under --window -1, --engine 4, ...)."""
    return (f"{cfg}/{dtype}/engine{plan['engine']}/launches{plan['launches']}/window{sel_opts.get('window', 0)}"
            f"/tma{sel_opts.get('tma', 0)}")


def load_traffic(key, q):
    """dram bytes (read + write) of launch q of the select identified by `key` (plan_key), from the
    committed ncu launch list of the same plan (profiles/traffic.json, written by
    tools/make_profiles.py from `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum`): the
    second select of the list (warm), else the first. None if that plan was not captured."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(p) as f:
            d = json.load(f).get(key)
        if not d:
            return None
        n = d["launches_per_select"]
        v = d["bytes"][n + q] if len(d["bytes"]) > n + q else d["bytes"][q]
        return float(v)
    except Exception:
        return None


def _timed(fn, steps, flush=None):
    """Mean device time of fn() over `steps` calls, CUDA events around each call on the current
    stream, L2 flushed (a 256 MB write) before each call when `flush` is given."""
    import torch
    tot = 0.0
    for _ in range(steps):
        if flush is not None:
            flush.fill_(1)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        tot += e0.elapsed_time(e1)
    return tot / steps


def per_rank_proxies(dev, steps=100):
    """What one rank of the 2/4/8-GPU runs does, measured on this one GPU: c2's
    row shards (50 / 25 / 13 rows of 2^20 normal keys, K = 256; no collective) and c5's per-rank
    work (the local select of a 2^30 uniform shard with K = 2^16, and the merge select over the
    8 x 2^16 gathered candidates; the NCCL all-gather between them is not in these numbers)."""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    peak, _ = hbm_peak()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    out = {}
    c = CFG["c2"]
    xh = host_keys("c2", c["n"], 50)
    x50 = torch.from_numpy(xh).to(dev)
    for rows in (50, 25, 13):
        x = x50[:rows].contiguous()
        ws = torch.empty(max(1, at.workspace_bytes(torch.float32, rows, c["n"], c["k"])), dtype=torch.uint8, device=dev)
        o = (torch.empty((rows, c["k"]), dtype=torch.float32, device=dev),
             torch.empty((rows, c["k"]), dtype=torch.int64, device=dev))
        fn = lambda: at.select(x, c["k"], workspace=ws, out=o)
        for _ in range(5):
            fn()
        ms = _timed(fn, steps, flush)
        alg = rows * c["n"] * 4 + rows * c["k"] * 12
        out[f"c2_rows{rows}"] = {"ms": ms, "elements_per_s": rows * c["n"] / (ms * 1e-3),
                                 "roofline_ms": alg / (peak * 1e9) * 1e3,
                                 "frac_of_peak": alg / (ms * 1e-3) / 1e9 / peak, "l2": "flushed"}
    del x50
    # c5 rank: local shard select (2^30 keys, global offset 0) + the 8 x 2^16 merge
    n, k, world = 1 << 30, 1 << 16, 8
    x = torch.from_numpy(host_keys("c5", n, 1)).to(dev).reshape(-1)
    ws = torch.empty(max(1, at.lib().airtopk_workspace_bytes_shard(at.dtype_code(torch.float32), n, k)),
                     dtype=torch.uint8, device=dev)
    o = (torch.empty(k, dtype=torch.float32, device=dev), torch.empty(k, dtype=torch.int64, device=dev))
    fn = lambda: at.select_shard(x, k, 0, (1 << 33), out=o, workspace=ws)
    for _ in range(3):
        fn()
    ms = _timed(fn, 20)
    alg = n * 4 + k * 12
    out["c5_shard_select"] = {"ms": ms, "elements_per_s": n / (ms * 1e-3), "roofline_ms": alg / (peak * 1e9) * 1e3,
                              "frac_of_peak": alg / (ms * 1e-3) / 1e9 / peak, "l2": "input > L2"}
    del x
    # merge input: 8 ranks' candidates = keys uniform on (0, 2^-14] (each shard's top 2^16 of 2^30
    # uniform (0,1] keys lies there) with distinct global indices r * 2^30 + j * 2^14
    m = world * k
    gv = torch.from_numpy(gen.uniform_f32(gen.config_seed("c5") + 1, m) * np.float32(2.0 ** -14)).to(dev)
    r = torch.arange(m, device=dev)
    gi = (r // k) * (1 << 30) + (r % k) * (1 << 14)
    bits = at.merge_idx_bits(1 << 33, world, k)
    wsm = torch.empty(max(1, at.lib().airtopk_workspace_bytes_with_idx(at.dtype_code(torch.float32), m, k, bits)),
                      dtype=torch.uint8, device=dev)
    mo = (torch.empty(k, dtype=torch.float32, device=dev), torch.empty(k, dtype=torch.int64, device=dev))
    fn = lambda: at.select_with_idx(gv, gi, k, bits, workspace=wsm, out=mo)
    for _ in range(5):
        fn()
    ms = _timed(fn, steps, flush)
    out["c5_merge_8x2^16"] = {"ms": ms, "elements_per_s": m / (ms * 1e-3), "l2": "flushed",
                              "input": "8 x 2^16 keys uniform on (0, 2^-14], distinct global indices"}
    return out


def extra_measure(name, dev, steps=None, warmup=5):
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    c = CFG[name]
    steps = steps or DEFAULT_STEPS[name]
    xh = host_keys(name, c["n"], c["batch"])
    xd = torch.from_numpy(xh).to(dev)
    k = c["k"]
    ws = torch.empty(max(1, at.workspace_bytes(torch.float32, c["batch"], c["n"], k)), dtype=torch.uint8, device=dev)
    ov = torch.empty((c["batch"], k), dtype=torch.float32, device=dev)
    oi = torch.empty((c["batch"], k), dtype=torch.int64, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    for _ in range(warmup):
        at.select(xd, k, workspace=ws, out=(ov, oi))
    torch.cuda.synchronize()
    small = c["batch"] * c["n"] * 4 < (512 << 20)
    tot = 0.0
    for _ in range(steps):
        if small:
            flush.fill_(1)  # write > L2 between timed iterations
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        at.select(xd, k, workspace=ws, out=(ov, oi))
        e1.record()
        e1.synchronize()
        tot += e0.elapsed_time(e1)
    ms = tot / steps
    in_bytes = c["batch"] * c["n"] * 4
    out_bytes = c["batch"] * k * 12
    peak, _ = hbm_peak()
    gbs = (in_bytes + out_bytes) / (ms * 1e-3) / 1e9
    return {"value": c["batch"] * c["n"] / (ms * 1e-3), "unit": "elements/s", "ms_per_step": ms,
            "alg_gbs": gbs, "frac_of_peak": gbs / peak, "steps": steps,
            "l2": "flushed (256 MB write) between steps" if small else "input > L2"}


if __name__ == "__main__":
    main()
