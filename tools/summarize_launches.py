"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list: per-kernel total time,
launch count and share of the summed device time (cold-cache, serialised: compare SHARES)."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hdr_i]
ik, im, iv = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[hdr_i + 1:]:
    if len(r) <= iv or r[im] != "gpu__time_duration.sum":
        continue
    name = r[ik].split("(")[0]
    if "k_gemm" in r[ik]:
        name = r[ik].split("(abft::GemmArgs")[0]
    tot[name] += float(r[iv].replace(",", ""))
    cnt[name] += 1
S = sum(tot.values())
print(f"{'kernel':70s} {'launches':>9s} {'total ms':>10s} {'share':>7s}")
for k in sorted(tot, key=lambda k: -tot[k]):
    print(f"{k[:70]:70s} {cnt[k]:9d} {tot[k]/1e6:10.3f} {tot[k]/S*100:6.2f}%")
print(f"{'TOTAL':70s} {sum(cnt.values()):9d} {S/1e6:10.3f}")
