"""Compact per-SASS-instruction dump of an `ncu --page source --csv --print-source sass` file:
index, executed warp instructions, stall samples, shared wavefronts, SASS text."""
import csv, sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
tot = 0
out = []
for k, r in enumerate(rows[2:]):
    if len(r) < len(hdr):
        continue
    ex = int(r[ix["Instructions Executed"]] or 0)
    smp = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    wf = int(r[ix["L1 Wavefronts Shared"]] or 0)
    tot += ex
    out.append((k, ex, smp, wf, r[ix["Source"]].strip()))
for k, ex, smp, wf, s in out:
    print(f"{k:5d} {ex:10d} {smp:6d} {wf:9d}  {s}")
print("total", tot, file=sys.stderr)
