"""NEXT-1, the paper's Fig. 8 analog (L2 and DRAM transactions of Fused normalised
to cuBLAS-Unfused): sum ncu's per-kernel dram / L2 byte counters over the kernels of ONE
timed step of each design (tools/fig8_step.py under
`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum`).

    python tools/fig8.py fused.csv unfused.csv [--md out.md]

The captures hold exactly one step each (tools/fig8_step.py, NVTX range "measured")."""
import csv
import sys
from collections import defaultdict

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-9, "us": 1e-6, "ms": 1e-3,
        "nsecond": 1e-9, "usecond": 1e-6,
        "msecond": 1e-3, "second": 1.0}


def load(path):
    rows = list(csv.DictReader(l for l in open(path) if not l.startswith("==")))
    per = defaultdict(lambda: defaultdict(list))
    for r in rows:
        try:
            v = float(r["Metric Value"].replace(",", "")) * UNIT.get(r["Metric Unit"], 1.0)
        except (KeyError, ValueError):
            continue
        per[(r["ID"], r["Kernel Name"])][r["Metric Name"]].append(v)
    launches = []
    for (i, name), m in per.items():
        launches.append((int(i), name, {k: v[0] for k, v in m.items()}))
    return sorted(launches)


def summarise(launches, keep):
    tot = defaultdict(float)
    names = defaultdict(int)
    for _, name, m in launches:
        if keep(name):
            names[name.split("(")[0][:70]] += 1
            for k, v in m.items():
                tot[k] += v
    return tot, names


if __name__ == "__main__":
    fused, unfused = load(sys.argv[1]), load(sys.argv[2])   # captures of one step each (NVTX "measured")
    tf, nf = summarise(fused, lambda n: True)
    tu, nu = summarise(unfused, lambda n: True)
    keys = ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "gpu__time_duration.sum"]
    out = ["| quantity (one step) | fused | unfused (SGEMM + one pass) | fused / unfused |", "|---|---|---|---|"]
    for k in keys:
        f, u = tf.get(k, 0.0), tu.get(k, 0.0)
        unit, sc = ("ms", 1e3) if "time" in k else ("GB", 1e-9)
        out.append(f"| {k} | {f * sc:.4g} {unit} | {u * sc:.4g} {unit} | {f / u if u else float('nan'):.2e} |")
    dram_f = tf["dram__bytes_read.sum"] + tf["dram__bytes_write.sum"]
    dram_u = tu["dram__bytes_read.sum"] + tu["dram__bytes_write.sum"]
    out.append(f"| DRAM bytes (read + write) | {dram_f * 1e-9:.4g} GB | {dram_u * 1e-9:.4g} GB | {dram_f / dram_u:.2e} |")
    out.append("")
    out.append("fused launches: " + ", ".join(f"{k} x{v}" for k, v in sorted(nf.items())))
    out.append("unfused launches: " + ", ".join(f"{k} x{v}" for k, v in sorted(nu.items())))
    out.append("(ncu serialises launches and runs them with cold caches: durations are per-kernel sums, not the step time)")
    text = "\n".join(out)
    print(text)
    if "--md" in sys.argv:
        open(sys.argv[sys.argv.index("--md") + 1], "w").write(text + "\n")
