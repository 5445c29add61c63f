"""Summarise `ncu --page source --csv --print-source cuda,sass` output: top CUDA lines by stall samples."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out, cur, hdr = [], None, None
for r in rows:
    if len(r) == 2 and r[0] in ("File Path", "File Name"):
        cur = r[1]; hdr = None; continue
    if r and r[0] == "Line No":
        hdr = r; continue
    if hdr and len(r) == len(hdr) and cur:
        d = dict(zip(hdr, r)); d["file"] = cur; out.append(d)
def f(x):
    try: return float(x)
    except: return 0.0
key = "Warp Stall Sampling (All Samples)"
tot = sum(f(d[key]) for d in out) or 1
stalls = [h for h in (hdr or []) if h.startswith("stall_") and "Not Issued" not in h]
for d in sorted(out, key=lambda d: -f(d[key]))[:n]:
    top = sorted(((f(d[s]), s[6:]) for s in stalls), reverse=True)[:3]
    print(f"{f(d[key])/tot*100:5.1f}% {d['file'].split('/')[-1]}:{d['Line No']:>4} inst={d['Instructions Executed']:>10} "
          f"[{', '.join(f'{k}:{v:.0f}' for v, k in top)}] {d['Source'][:80]}")
