"""Write profiles/ summaries from ncu outputs: per-kernel-class traffic table + full-capture key metrics,
and profiles/ncu_traffic.json (dram bytes per launch of the conv GEMM) read by bench.py."""
import csv, json, subprocess, sys
tag = sys.argv[1]
traffic_csv, full_rep = sys.argv[2], sys.argv[3]
rows = list(csv.reader(open(traffic_csv)))
hdr, data = None, {}
for r in rows:
    if "Kernel Name" in r:
        hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        data.setdefault(d["ID"], {"name": d["Kernel Name"].split("(")[0]})[d["Metric Name"]] = d["Metric Value"]
def f(x):
    try: return float(x)
    except: return 0.0
cls = {}
for d in data.values():
    k = d["name"]
    c = cls.setdefault(k, [0, 0.0, 0.0, 0.0, 0.0])
    c[0] += 1
    c[1] += f(d.get("gpu__time_duration.sum"))
    c[2] += f(d.get("dram__bytes_read.sum")) + f(d.get("dram__bytes_write.sum"))
    c[3] += f(d.get("sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed")) * f(d.get("gpu__time_duration.sum"))
tot_t = sum(c[1] for c in cls.values())
out = [f"# {tag}: one ResNet-18-EE step (infer 256 + retrain 1024), ncu launch metrics (cold, serialised: "
       f"compare shares, not absolutes)\n",
       "| kernel | launches | time ms | share | DRAM GB | avg GB/s | tensor-pipe % (time-weighted) |",
       "|---|---|---|---|---|---|---|"]
for k, c in sorted(cls.items(), key=lambda kv: -kv[1][1]):
    if c[1] < 0.005 * tot_t: continue
    unit = 1e9 if max(c[2], 1) > 1e6 else 1.0
    out.append(f"| `{k[:60]}` | {c[0]} | {c[1]/1e6:.3f} | {c[1]/tot_t*100:.1f}% | {c[2]/1e9:.3f} | "
               f"{c[2]/max(c[1],1):.0f} | {c[3]/max(c[1],1):.1f} |")
conv = [d for d in data.values() if d["name"].startswith(("void conv_", "conv_"))]
conv_bytes = sum(f(d.get("dram__bytes_read.sum")) + f(d.get("dram__bytes_write.sum")) for d in conv)
conv_t = sum(f(d.get("gpu__time_duration.sum")) for d in conv)
out.append(f"\nconv GEMM (all variants): {len(conv)} launches, {conv_t/1e6:.3f} ms, DRAM {conv_bytes/1e9:.3f} GB "
           f"({conv_bytes/max(len(conv),1)/1e6:.1f} MB per launch), share {conv_t/tot_t*100:.1f}% of kernel time\n")
json.dump({"tag": tag, "conv_umma_kernel_bytes_per_launch": conv_bytes / max(len(conv), 1),
           "conv_launches": len(conv), "conv_time_ms": conv_t / 1e6, "source": traffic_csv},
          open("profiles/ncu_traffic.json", "w"), indent=1)
# full capture: key metrics per profiled kernel
raw = open(full_rep).read() if full_rep.endswith(".csv") else subprocess.run(
    ["ncu", "-i", full_rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(raw.splitlines()))
h = rr[0]
keys = ["gpu__time_duration.sum", "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "lts__t_sectors.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active"]
out.append("## ncu --set full captures (key metrics)\n")
out.append("| kernel | " + " | ".join(k.split(".")[-3] if k.startswith("TPC") else k for k in keys) + " |")
out.append("|---|" + "---|" * len(keys))
for row in rr[2:]:
    d = dict(zip(h, row))
    out.append(f"| `{d.get('Kernel Name','')[:50]}` | " + " | ".join(d.get(k, "") for k in keys) + " |")
open(f"profiles/{tag}_summary.md", "w").write("\n".join(out) + "\n")
print("\n".join(out))
