"""Summarise an ncu --csv launch list (gpu__time_duration.sum [+ tensor pipe %])."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 100.0
hdr, data = None, {}
for r in rows:
    if "Kernel Name" in r:
        hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        data.setdefault(d["ID"], {"name": d["Kernel Name"], "grid": d["Grid Size"]})[d["Metric Name"]] = d["Metric Value"]
def f(x):
    try: return float(x)
    except: return 0.0
tot = 0
byname = {}
for i, d in sorted(data.items(), key=lambda kv: int(kv[0])):
    t = f(d.get("gpu__time_duration.sum")); tot += t
    k = d["name"].split("(")[0]
    byname[k] = byname.get(k, 0) + t
    if t > thr * 1e3:
        tc = d.get("sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "")
        print(f"{i:>4} {t/1e3:9.1f}us tc={tc:>6} {d['grid']:>12} {d['name'][:50]}")
print("total ms", tot / 1e6)
for k, v in sorted(byname.items(), key=lambda kv: -kv[1])[:12]:
    print(f"  {v/1e6:8.3f} ms  {k[:70]}")
