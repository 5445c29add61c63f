"""Per-launch table of one profiled step from an ncu --csv launch list (time us, DRAM MB read/write)."""
import csv, io, sys, collections
lines = open(sys.argv[1]).read().splitlines()
i = [k for k, l in enumerate(lines) if l.startswith('"ID"')][0]
rows = list(csv.DictReader(io.StringIO("\n".join(lines[i:]))))
per = collections.OrderedDict()
for r in rows:
    key = (int(r['ID']), r['Kernel Name'][:38], r['Grid Size'])
    try:
        per.setdefault(key, {})[r['Metric Name']] = float(r['Metric Value'].replace(',', '') or 0)
    except ValueError:
        per.setdefault(key, {})
ids = sorted(set(k[0] for k in per))
lo = int(sys.argv[2]) if len(sys.argv) > 2 else 0
tot = 0
for (id_, name, g), m in per.items():
    if id_ < lo: continue
    t = m['gpu__time_duration.sum'] / 1e3
    tot += t
    print(f"{id_:4d} {name:38s} {g:14s} {t:8.1f} {m.get('dram__bytes_read.sum',0)/1e6:7.0f} {m.get('dram__bytes_write.sum',0)/1e6:7.0f}")
print("total us", tot)
