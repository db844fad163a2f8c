"""Copy the judged evidence of one GPU round from gpurun_out/<tag> into
profiles/<round>/ (tracked): ncu summaries (text), launch list summary, bench
JSON lines; update profiles/ncu_summary.json (DRAM bytes per fused launch, read
by bench.py as roofline.traffic)."""
import csv, io, json, os, shutil, subprocess, sys

tag, rnd = sys.argv[1], sys.argv[2]
cfgs = sys.argv[3:] or ["3"]   # entries like "3" or "4" (auto path) or "3_3xtf32"
src = os.path.join("gpurun_out", tag)
dst = os.path.join("profiles", rnd)
os.makedirs(dst, exist_ok=True)
summ_path = os.path.join("profiles", "ncu_summary.json")
summ = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
for c in cfgs:   # "3", "4", "3_fp32", ... -> prof_cfg<c>.ncu-rep
    rep = os.path.join(src, f"prof_cfg{c}.ncu-rep")
    if os.path.exists(rep):
        out = subprocess.run([sys.executable, "tools/ncu_summary.py", rep], capture_output=True, text=True).stdout
        open(os.path.join(dst, f"ncu_full_fused_cfg{c}.txt"), "w").write(
            f"# ncu --set full --clock-control none, fused kernel, cfg{c} (from {rep})\n" + out)
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(raw)))
        d = dict(zip(rows[0], rows[2])); u = dict(zip(rows[0], rows[1]))
        def b(k):
            v = float(d[k].replace(",", "")); s = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u[k]]
            return v * s
        summ[f"cfg{c}"] = {"kernel": rows[2][rows[0].index("Kernel Name")] if "Kernel Name" in rows[0] else "ks_fused",
                           "dram_bytes_per_launch": b("dram__bytes_read.sum") + b("dram__bytes_write.sum"),
                           "source": f"profiles/{rnd}/ncu_full_fused_cfg{c}.txt"}
for f in ("launches.csv",):
    p = os.path.join(src, f)
    if os.path.exists(p):
        out = subprocess.run([sys.executable, "tools/launch_summary.py", p], capture_output=True, text=True).stdout
        open(os.path.join(dst, "launches_summary.txt"), "w").write(
            "# ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised) of\n"
            "# python bench.py --steps 2 --warmup 3 --no-cpu-baseline\n" + out)
        shutil.copy(p, os.path.join(dst, "launches.csv"))
for f in os.listdir(src):
    if f.startswith("bench") and f.endswith(".json"):
        shutil.copy(os.path.join(src, f), os.path.join(dst, f))
json.dump(summ, open(summ_path, "w"), indent=1)
print("wrote", dst, summ)
