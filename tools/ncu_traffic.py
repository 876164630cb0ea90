"""Per-launch DRAM traffic of one kernel from an ncu CSV (metrics dram__bytes_read.sum,
dram__bytes_write.sum, gpu__time_duration.sum), written as JSON for bench.py's roofline.traffic.
usage: python tools/ncu_traffic.py launches.csv out.json "command that was profiled" """
import csv
import json
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hdr_i]
iid, ik, im, iu, iv = (hdr.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
         "nsecond": 1e-9, "msecond": 1e-3, "ms": 1e-3}
per = defaultdict(dict)
name = None
for r in rows[hdr_i + 1:]:
    if len(r) <= iv:
        continue
    per[r[iid]][r[im]] = float(r[iv].replace(",", "")) * scale.get(r[iu], 1.0)
    name = r[ik].split("(abft::GemmArgs")[0]
L = [v for v in per.values() if "dram__bytes_read.sum" in v]
rd = sum(v["dram__bytes_read.sum"] for v in L)
wr = sum(v["dram__bytes_write.sum"] for v in L)
t = sum(v.get("gpu__time_duration.sum", 0.0) for v in L)
out = {"kernel": name, "launches": len(L), "dram_read_bytes": rd, "dram_write_bytes": wr,
       "traffic_bytes_per_launch": (rd + wr) / max(1, len(L)), "device_seconds_serialised": t,
       "command": sys.argv[3] if len(sys.argv) > 3 else ""}
json.dump(out, open(sys.argv[2], "w"), indent=1)
print(json.dumps(out, indent=1))
