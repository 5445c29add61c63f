"""Round-2 profiles/ summary from one tools/profile_r2.sh run: bench lines (c5 / c2 / c3), the bench launch list
(cold, serialised: shares, not absolutes), per-class DRAM traffic of a C5-shaped step, and key metrics of the
ncu --set full captures.  usage: python tools/summarize_r2.py TAG"""
import csv, json, os, shutil, sys
tag = sys.argv[1]
G = "gpurun_out"


def f(x):
    try:
        return float(x)
    except Exception:
        return 0.0


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, {}
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            data.setdefault(d["ID"], {"name": d["Kernel Name"].split("(")[0]})[d["Metric Name"]] = d["Metric Value"]
    return data


out = [f"# {tag}: round-2 profile (B200, `tools/profile_r2.sh {tag}`)\n", "## Bench lines (no profiler)\n",
       "| config | value | unit | ms/step | e2e | roofline frac (dominant class) | clocks |", "|---|---|---|---|---|---|---|"]
for c in ("c5", "c2", "c3"):
    p = f"{G}/{tag}_bench_{c}.json"
    if not os.path.exists(p) or os.path.getsize(p) == 0:
        continue
    d = json.load(open(p))
    rf = d.get("roofline") or {}
    out.append(f"| {c} | {d['value']:.0f} | {d['unit']} | {d['ms_per_step']:.2f} | {d.get('e2e', {}).get('value', 0):.0f} | "
               f"{rf.get('frac', 0):.3f} vs {rf.get('peak_kind', '')[:40]} | {d.get('clocks', {}).get('sm_mhz')} MHz "
               f"{d.get('clocks', {}).get('reasons')} |")
    shutil.copy(p, f"profiles/{tag}_bench_{c}.json")
p = f"{G}/{tag}_bench_launch_list.csv"
if os.path.exists(p):
    data = launches(p)
    tot = sum(f(d.get("gpu__time_duration.sum")) for d in data.values())
    cls = {}
    for d in data.values():
        c = cls.setdefault(d["name"], [0, 0.0])
        c[0] += 1
        c[1] += f(d.get("gpu__time_duration.sum"))
    out += ["\n## Launch list of `python bench.py --steps 1 --warmup 3` (C5; gpu__time_duration, cold + serialised)\n",
            f"{len(data)} launches, {tot / 1e6:.2f} ms in total (warm-up + calibration + the timed step)\n",
            "| kernel | launches | ms | share |", "|---|---|---|---|"]
    for k, c in sorted(cls.items(), key=lambda kv: -kv[1][1])[:25]:
        out.append(f"| `{k[:70]}` | {c[0]} | {c[1] / 1e6:.3f} | {c[1] / tot * 100:.1f}% |")
    shutil.copy(p, f"profiles/{tag}_bench_launch_list.csv")
p = f"{G}/{tag}_c3_launch_list.csv"
if os.path.exists(p):
    data = launches(p)
    steps = max(1, sum(1 for d in data.values() if d["name"].startswith("void adainf::det_count_kernel")
                       or d["name"].startswith("adainf::det_count_kernel")))
    cls = {}
    for d in data.values():
        c = cls.setdefault(d["name"], [0, 0.0, 0.0])
        c[0] += 1
        c[1] += f(d.get("gpu__time_duration.sum"))
        c[2] += f(d.get("dram__bytes_read.sum")) + f(d.get("dram__bytes_write.sum"))
    tot = sum(c[1] for c in cls.values())
    out += [f"\n## C3 (`bench.py --config c3 --steps 1 --warmup 3`): per-class time and DRAM traffic per DAG step "
            f"(ncu, cold + serialised; {steps} detector passes in the run, totals divided by that)\n",
            "| kernel | launches/step | ms/step | share | DRAM GB/step | GB/s |", "|---|---|---|---|---|---|"]
    for k, c in sorted(cls.items(), key=lambda kv: -kv[1][1])[:24]:
        out.append(f"| `{k[:70]}` | {c[0] / steps:.1f} | {c[1] / 1e6 / steps:.3f} | {c[1] / tot * 100:.1f}% | "
                   f"{c[2] / 1e9 / steps:.3f} | {c[2] / max(c[1], 1):.0f} |")
    shutil.copy(p, f"profiles/{tag}_c3_launch_list.csv")
p = f"{G}/{tag}_step_traffic.csv"
if os.path.exists(p):
    data = launches(p)
    tot = sum(f(d.get("gpu__time_duration.sum")) for d in data.values())
    cls = {}
    for d in data.values():
        c = cls.setdefault(d["name"], [0, 0.0, 0.0, 0.0])
        c[0] += 1
        t = f(d.get("gpu__time_duration.sum"))
        c[1] += t
        c[2] += f(d.get("dram__bytes_read.sum")) + f(d.get("dram__bytes_write.sum"))
        c[3] += f(d.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed")) * t
    out += ["\n## One C5-shaped step (infer 256 + retrain 8,192), per-class DRAM traffic and tensor-pipe activity "
            "(ncu, cold + serialised)\n",
            "| kernel | launches | ms | share | DRAM GB | GB/s | tensor pipe % (time-weighted) |",
            "|---|---|---|---|---|---|---|"]
    for k, c in sorted(cls.items(), key=lambda kv: -kv[1][1])[:25]:
        out.append(f"| `{k[:70]}` | {c[0]} | {c[1] / 1e6:.3f} | {c[1] / tot * 100:.1f}% | {c[2] / 1e9:.3f} | "
                   f"{c[2] / max(c[1], 1):.0f} | {c[3] / max(c[1], 1):.1f} |")
    shutil.copy(p, f"profiles/{tag}_step_traffic.csv")
keys = ["gpu__time_duration.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__ops_path_tensor_src_bf16_dst_fp32.avg.pct_of_peak_sustained_elapsed", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size"]
out += ["\n## ncu --set full captures (one launch each)\n",
        "| kernel | " + " | ".join(k.replace(".avg.pct_of_peak_sustained", "%").replace("sm__", "") for k in keys) + " |",
        "|---|" + "---|" * len(keys)]
for fn in sorted(os.listdir(G)):
    if not (fn.startswith(tag + "_") and fn.endswith("_raw.csv")) or os.path.getsize(f"{G}/{fn}") < 1000:
        continue
    rr = list(csv.reader(open(f"{G}/{fn}")))
    h = rr[0]
    for row in rr[2:]:
        d = dict(zip(h, row))
        out.append(f"| `{d.get('Kernel Name', '')[:48]}` | " + " | ".join(d.get(k, "") for k in keys) + " |")
    shutil.copy(f"{G}/{fn}", f"profiles/{fn}")
open(f"profiles/{tag}_summary.md", "w").write("\n".join(out) + "\n")
print("\n".join(out))
