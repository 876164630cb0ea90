"""Summarise an ncu launch list (metrics gpu__time_duration.sum [+ dram__bytes_read.sum,
dram__bytes_write.sum]): per-kernel launches, total time, share of the summed device time and,
when the DRAM metrics are present, achieved DRAM GB/s (cold-cache, serialised replay: compare
SHARES for the step, and GB/s for each kernel standalone).
usage: python tools/summarize_launches.py launches.csv"""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hdr_i]
iid, ik, im, iu, iv = (hdr.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "ns": 1, "usecond": 1e3, "us": 1e3,
         "msecond": 1e6, "ms": 1e6}
per = defaultdict(dict)
names = {}
for r in rows[hdr_i + 1:]:
    if len(r) <= iv:
        continue
    name = r[ik].split("(")[0]
    if "k_gemm" in r[ik] or "k_update" in r[ik]:
        name = r[ik].split("(abft::GemmArgs")[0].split("(GemmArgs")[0]
    names[r[iid]] = name
    per[r[iid]][r[im]] = float(r[iv].replace(",", "")) * scale.get(r[iu], 1.0)
tot, cnt, byt = defaultdict(float), defaultdict(int), defaultdict(float)
for i, m in per.items():
    k = names[i]
    tot[k] += m.get("gpu__time_duration.sum", 0.0)
    cnt[k] += 1
    byt[k] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
S = sum(tot.values())
print(f"{'kernel':64s} {'launches':>8s} {'total ms':>9s} {'share':>7s} {'DRAM GB':>8s} {'GB/s':>7s}")
for k in sorted(tot, key=lambda k: -tot[k]):
    gbs = byt[k] / tot[k] if tot[k] else 0.0   # bytes / ns = GB/s
    print(f"{k[:64]:64s} {cnt[k]:8d} {tot[k]/1e6:9.3f} {tot[k]/S*100:6.2f}% {byt[k]/1e9:8.2f} {gbs:7.0f}")
print(f"{'TOTAL':64s} {sum(cnt.values()):8d} {S/1e6:9.3f}")
