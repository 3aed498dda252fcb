"""Print an ncu --metrics --csv launch list as one line per launch."""
import csv
import sys

for f in sys.argv[1:]:
    rows = [r for r in csv.reader(open(f)) if len(r) > 10]
    h = rows[0]
    ik, im, iv, iid = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value'), h.index('ID')
    d = {}
    for r in rows[1:]:
        d.setdefault((int(r[iid]), r[ik].split('(')[0][-40:]), {})[r[im]] = r[iv]
    print(f)
    for k, v in sorted(d.items()):
        print(k, {a.split('.')[0][:24]: v[a] for a in sorted(v)})
