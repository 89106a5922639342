import glob, json, sys, os
rows = []
for f in sorted(glob.glob("gpurun_out/ab_*.json")):
    try:
        d = json.load(open(f))
    except Exception as e:
        print(os.path.basename(f), "ERR", open(f.replace(".json", ".err")).read()[-300:]); continue
    pk = d["whole_select"]["per_kernel_ms"]
    print(f"{os.path.basename(f):32s} {d['ms_per_step']:.4f} ms  kernels " + " ".join(f"{x*1e3:.1f}" for x in pk), d["plan"]["ctas_per_row"], d["clocks"]["sm_mhz"])
