"""Summarise gpurun_out/ab_env.jsonl (tools/ab_env.sh): median on/off ms per (n, env)."""
import collections, json, statistics, sys
rows = collections.defaultdict(lambda: ([], []))
for line in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ab_env.jsonl"):
    d = json.loads(line)
    key = (d["n"], d["nb"], json.dumps({k: v for k, v in d["env"].items() if k != "ABFT_DEV_ABLATE"}, sort_keys=True))
    rows[key][0].extend(d["on_ms"]); rows[key][1].extend(d["off_ms"])
for (n, nb, env), (on, off) in sorted(rows.items()):
    mon, moff = statistics.median(on), statistics.median(off)
    print(f"n={n:6d} nb={nb:4d} {env:40s} on {mon:9.3f} ms ({n**3/3/mon/1e9:7.1f} TF/s)  off {moff:9.3f} ms  overhead {100*(mon-moff)/moff:5.2f} %")
