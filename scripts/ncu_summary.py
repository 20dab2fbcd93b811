"""Summarise gpurun_out/launches.csv (ncu launch list) and gpurun_out/prof_full.ncu-rep
(ncu --set full) into a markdown table on stdout (needs ncu on PATH; no GPU)."""
import collections
import csv
import subprocess
import sys

out = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out"
rows = list(csv.reader(open(f"{out}/launches.csv")))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
agg = collections.defaultdict(list)
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    v = float(r[vi].replace(",", ""))
    v *= {"usecond": 1e3, "msecond": 1e6}.get(r[ui], 1.0)
    agg[r[ki].split("(")[0].replace("void ", "")].append(v)
tot = sum(sum(v) for v in agg.values())
print("| kernel | launches | ns / launch | share |\n|---|---:|---:|---:|")
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
    print(f"| {k} | {len(v)} | {sum(v) / len(v):,.0f} | {100 * sum(v) / tot:.1f} % |")
mets = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__cycles_elapsed.avg.per_second", "launch__registers_per_thread", "smsp__inst_executed.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]
r = subprocess.run(["ncu", "-i", f"{out}/prof_full.ncu-rep", "--page", "raw", "--csv", "--metrics", ",".join(mets)],
                   capture_output=True, text=True).stdout
rr = list(csv.reader(r.splitlines()))
h = rr[0]
print("\n| kernel | time (ms) | SM GHz | DRAM R + W (GB) | DRAM % | SM % | tensor % | regs | warp-instr (M) |")
print("|---|---:|---:|---:|---:|---:|---:|---:|---:|")
for row in rr[2:]:
    d = dict(zip(h, row))
    f = lambda m: float(d.get(m, "0").replace(",", "") or 0)  # noqa: E731
    print(f"| {d['Kernel Name'].split('(')[0].replace('void ', '')} | {f(mets[0]):.3f} | {f(mets[5]):.2f} | "
          f"{f(mets[1]):.3f} + {f(mets[2]):.3f} | {f(mets[8]):.1f} | {f(mets[3]):.1f} | {f(mets[4]):.1f} | "
          f"{f(mets[6]):.0f} | {f(mets[7]) / 1e6:.0f} |")
