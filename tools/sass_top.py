"""Top SASS instructions by warp-stall samples from `ncu --page source --csv --print-source sass`."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
hdr = rows[1]
out = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
def f(x):
    try: return float(x)
    except: return 0.0
key = "Warp Stall Sampling (All Samples)"
tot = sum(f(d[key]) for d in out) or 1
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
print("total samples", tot, "instructions", len(out))
for i, d in sorted(enumerate(out), key=lambda x: -f(x[1][key]))[:n]:
    top = sorted(((f(d[s]), s[6:]) for s in stalls), reverse=True)[:3]
    print(f"{f(d[key])/tot*100:5.1f}% #{i:5d} ex={d['Instructions Executed']:>9} [{', '.join(f'{k}:{v:.0f}' for v, k in top)}] {d['Source'][:90]}")
