"""Summarise an ncu --csv launch list: per kernel name, count and mean time (µs)."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = None
agg = collections.OrderedDict()
seq = []
for r in rows:
    if r and r[0] == 'ID':
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d['Metric Name'] == 'gpu__time_duration.sum':
            v = float(d['Metric Value'].replace(',', ''))
            if d['Metric Unit'] == 'ms': v *= 1e3
            elif d['Metric Unit'] in ('ns', 'nsecond'): v /= 1e3
            seq.append((d['Kernel Name'].split('(')[0][-50:], v))
for name, v in seq:
    print(f"{v:10.1f} us  {name}")
