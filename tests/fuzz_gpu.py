"""Randomised GPU-vs-oracle fuzzing (not collected by pytest; run on a GPU box):

    python tests/fuzz_gpu.py SECONDS [SEED]

Random key type, batch, length (edges favoured), K, direction, value pattern (uniform bits, few
distinct values, shared leading bits, sorted / reversed, special values), engine, window, alpha,
early stop. Every case is compared bit-exactly with the CPU oracle (helpers.assert_parity).
Prints one line per failure and a summary; exit code 1 on any failure."""
import os
import sys
import time
import traceback

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))

import gen  # noqa: E402
from helpers import assert_parity, gpu_select  # noqa: E402

BITS = {"f32": np.uint32, "f16": np.uint16, "bf16": np.uint16, "f64": np.uint64, "u32": np.uint32}


def make_keys(rng, dtn, batch, n):
    nb = np.dtype(BITS[dtn]).itemsize * 8
    total = batch * n
    u = gen.u64(int(rng.integers(1 << 30)), total)
    pat = rng.choice(["bits", "few", "prefix", "sorted", "reversed", "special", "floats"])
    if pat == "few":
        pool = gen.u64(int(rng.integers(1 << 30)), int(rng.integers(1, 8)))
        u = pool[u % np.uint64(pool.size)]
    elif pat == "prefix":
        keep = int(rng.integers(1, nb))
        base = np.uint64(int(rng.integers(0, 1 << 62)))
        mask = np.uint64((1 << keep) - 1)
        u = (base & ~mask) | (u & mask)
    raw = u.astype(BITS[dtn])
    if pat == "floats" and dtn in ("f32", "f64", "f16"):
        ft = {"f32": np.float32, "f64": np.float64, "f16": np.float16}[dtn]
        raw = (rng.standard_normal(total) * 10 ** rng.uniform(-3, 3)).astype(ft).view(BITS[dtn])
    if pat == "special" and dtn in ("f32",):
        sp = np.array([0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000, 0xFFC00001, 0x00000001,
                       0x3F800000], dtype=np.uint32)
        raw = sp[u % np.uint64(sp.size)]
    raw = raw.reshape(batch, n)
    if pat in ("sorted", "reversed"):
        raw = np.sort(raw, axis=1)
        if pat == "reversed":
            raw = raw[:, ::-1].copy()
    return raw, pat


def main():
    seconds = float(sys.argv[1]) if len(sys.argv) > 1 else 60.0
    seed = int(sys.argv[2]) if len(sys.argv) > 2 else 12345
    rng = np.random.default_rng(seed)
    t0 = time.time()
    cases = fails = 0
    while time.time() - t0 < seconds:
        dtn = str(rng.choice(["f32", "f32", "f16", "bf16", "f64", "u32"]))
        r = rng.random()
        if r < 0.3:
            n = int(rng.integers(1, 300))
        elif r < 0.7:
            n = int(rng.integers(300, 1 << 17))
        else:
            n = int(rng.integers(1 << 17, 1 << 21))
        batch = int(rng.choice([1, 1, 1, 2, 3, 7, 33, 150])) if n < (1 << 18) else int(rng.choice([1, 1, 4, 20]))
        k = int(rng.choice([1, 2, max(1, n // 1000), max(1, n // 10), n // 2 + 1, n, int(rng.integers(1, n + 1))]))
        k = max(1, min(k, n))
        sm = bool(rng.integers(0, 2))
        kw = {}
        engine = int(rng.choice([0, 0, 1, 2, 4, 5, 6, 7]))
        if engine in (4, 7) and (dtn == "f64" or k > 2048):
            engine = 0
        if engine:
            kw["engine"] = engine
        if engine in (0, 1) and rng.random() < 0.5:
            kw["window"] = int(rng.choice([-1, 1]))
        if rng.random() < 0.3:
            kw["alpha"] = int(rng.choice([1, 4, 128, 1 << 40]))
        if rng.random() < 0.2:
            kw["early_stop"] = -1
        if engine in (2, 6) and rng.random() < 0.5:
            kw["cluster_size"] = int(rng.choice([1, 2, 4, 8, 16]))
        if rng.random() < 0.1 and k <= 4096:
            kw["sorted"] = True
        abl = rng.random() < 0.05 and dtn != "f64" and k < n
        raw, pat = make_keys(rng, dtn, batch, n)
        cases += 1
        try:
            if abl:  # the paper's kernel organisations (ablation harness)
                import torch
                import paper_conf_sc_zhangnlw23_b200 as at
                from helpers import to_bits, to_device
                design, b = int(rng.integers(0, 3)), int(rng.choice([8, 11]))
                kw = {"ablation": (design, b)}
                vv, ii, _ = at.select_ablation(to_device(raw, dtn), k, design, b, largest=not sm)
                torch.cuda.synchronize()
                v, i = to_bits(vv, dtn), ii.cpu().numpy()
            else:
                try:
                    v, i = gpu_select(raw, dtn, k, sm, **kw)
                except Exception as e:  # an engine the shape is not eligible for: AIRTOPK_EINVAL
                    if kw.get("engine") in (5, 6) and "EINVAL" in str(e):
                        cases -= 1
                        continue
                    raise
            assert_parity(raw, dtn, k, sm, v, i)
        except Exception as e:  # noqa: BLE001
            fails += 1
            print(f"FAIL dtn={dtn} batch={batch} n={n} k={k} min={sm} pat={pat} kw={kw}: {str(e)[:200]}", flush=True)
            if fails > 20:
                break
    print(f"fuzz: {cases} cases, {fails} failures, {time.time() - t0:.0f} s, seed {seed}", flush=True)
    sys.exit(1 if fails else 0)


if __name__ == "__main__":
    main()
