"""Summarise an ncu --set full report (run here, no GPU): key throughput
metrics + top stall reasons per SASS opcode/instruction."""
import csv, io, subprocess, sys
from collections import defaultdict

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
d = dict(zip(hdr, vals))
want = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__t_bytes.sum", "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__occupancy_limit_registers",
        "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_tc_wavefronts_mem_shared.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed"]
for k in want:
    if k in d:
        print(f"{k:70s} {d[k]:>16s} {units[hdr.index(k)]}")
print("stall reasons (per issued instruction):")
st = [(float(d[k]), k) for k in hdr if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio") and d[k] not in ("", "n/a")]
for v, k in sorted(st, reverse=True)[:10]:
    print(f"   {k.replace('smsp__average_warps_issue_stalled_','').replace('_per_issue_active.ratio',''):28s} {v:.3f}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = rows[1]; data = rows[2:]
iS = hdr.index("Source"); iN = hdr.index("Warp Stall Sampling (Not-issued Samples)"); iA = hdr.index("Warp Stall Sampling (All Samples)")
scols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" in h]
tot = sum(int(r[iA]) for r in data); totN = sum(int(r[iN]) for r in data)
print(f"samples: all {tot}, not-issued {totN}")
byop = defaultdict(lambda: [0, 0])
for r in data:
    t = r[iS].split()
    op = (t[1] if t and t[0].startswith("@") else (t[0] if t else "")).split(".")[0]
    byop[op][0] += int(r[iA]); byop[op][1] += int(r[iN])
print("by opcode (all, not-issued):", ", ".join(f"{o}:{a}/{n}" for o, (a, n) in sorted(byop.items(), key=lambda x: -x[1][1])[:12]))
reason_tot = defaultdict(int)
for r in data:
    for i in scols:
        if r[i] not in ("", "0"):
            reason_tot[hdr[i]] += int(r[i])
print("not-issued by reason:", ", ".join(f"{k.replace(' (Not Issued)','')}:{v}" for k, v in sorted(reason_tot.items(), key=lambda x: -x[1])[:8]))
top = sorted(data, key=lambda r: -int(r[iN]))[:12]
for r in top:
    rs = sorted([(int(r[i]), hdr[i].replace(" (Not Issued)", "")) for i in scols if r[i] not in ("0", "")], reverse=True)[:2]
    print(f"  {r[0][-5:]} {r[iS].strip()[:60]:60s} {r[iN]:>6s} {rs}")
