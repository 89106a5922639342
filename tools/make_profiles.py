"""Copy the judged evidence from gpurun_out/ (scratch) into profiles/ (tracked), named per round.

    python tools/make_profiles.py r01
Writes:
  profiles/<round>_launches_<cfg>.txt   per-launch device time + DRAM bytes (ncu, serialised, cold cache)
  profiles/<round>_ncu_<name>.txt       key metrics of each `ncu --set full` capture
  profiles/<round>_bench_<cfg>.json     bench.py JSON lines
  profiles/traffic.json                 dram bytes per launch for bench.py's roofline.traffic
"""
import csv
import glob
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import ncu_summary  # noqa: E402

OUT = os.path.join(ROOT, "gpurun_out")  # (a sub-directory may be given as the 2nd argument)
PROF = os.path.join(ROOT, "profiles")

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__sectors_read.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sectors_srcunit_tex_op_read.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "lts__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard.pct", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]


def main(rnd, out=OUT):
    global OUT
    OUT = out
    os.makedirs(PROF, exist_ok=True)
    tpath = os.path.join(PROF, "traffic.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}  # merged: plans not re-measured stay
    for f in sorted(glob.glob(os.path.join(OUT, "launches_*.csv"))):
        cfg = os.path.basename(f)[len("launches_"):-4]
        try:
            L = ncu_summary.load(f)
        except Exception as e:  # noqa: BLE001
            print("skip", f, e)
            continue
        lines = [f"# {cfg}: ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                 f"--clock-control none (serialised launches, cold cache: compare shares, not absolutes)",
                 f"{'#':>3} {'kernel':50s} {'time_us':>9} {'dram_read_MB':>12} {'dram_write_MB':>13}"]
        per = {}
        for i, d in enumerate(L):
            t = d.get("gpu__time_duration.sum", 0) / 1e3
            rd = d.get("dram__bytes_read.sum", 0)
            wr = d.get("dram__bytes_write.sum", 0)
            lines.append(f"{i:3d} {ncu_summary.short(d['name'])[:50]:50s} {t:9.1f} {rd / 1e6:12.1f} {wr / 1e6:13.1f}")
            per.setdefault(i, rd + wr)
        open(os.path.join(PROF, f"{rnd}_launches_{cfg}.txt"), "w").write("\n".join(lines) + "\n")
        side = os.path.join(OUT, f"plan_{cfg}.json")  # written by prof_select.py --plan-out
        if os.path.exists(side):
            pk = json.load(open(side))
            traffic[pk["plan_key"]] = {"launches_per_select": pk["launches_per_select"],
                                       "bytes": [per[i] for i in sorted(per)], "source": f"{rnd}_launches_{cfg}.txt"}
    for f in sorted(glob.glob(os.path.join(OUT, "*.ncu-rep"))):
        name = os.path.basename(f)[:-8]
        raw = subprocess.run(["ncu", "-i", f, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(raw)))
        if len(rows) < 3:
            continue
        h = rows[0]
        lines = [f"# ncu --set full capture {name} (key metrics; units as reported by ncu)"]
        for r in rows[2:]:
            lines.append(f"== {r[h.index('Kernel Name')][:100]}")
            for k in KEYS:
                if k in h:
                    lines.append(f"   {k:62s} {r[h.index(k)]} {rows[1][h.index(k)]}")
        open(os.path.join(PROF, f"{rnd}_ncu_{name}.txt"), "w").write("\n".join(lines) + "\n")
    for f in sorted(glob.glob(os.path.join(OUT, "bench_*.json"))):
        if "sanity" in f:
            continue
        txt = open(f).read().strip()
        if txt:
            open(os.path.join(PROF, f"{rnd}_{os.path.basename(f)}"), "w").write(txt.splitlines()[-1] + "\n")
    json.dump(traffic, open(tpath, "w"), indent=1)
    print("wrote", sorted(os.listdir(PROF)))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r02", sys.argv[2] if len(sys.argv) > 2 else OUT)
