"""Print the last N launches of an ncu --metrics gpu__time_duration.sum --csv launch list."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr, data = None, []
for r in rows:
    if r and r[0] == 'ID':
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d['Metric Name'] == 'gpu__time_duration.sum':
            data.append((int(d['ID']), d['Kernel Name'][:60], float(d['Metric Value']) / 1e3, d.get('Grid Size', ''),
                         d.get('Block Size', '')))
for x in data[-n:]:
    print(f"{x[0]:4d} {x[2]:8.2f} us  {x[3]:>14} {x[4]:>12}  {x[1]}")
