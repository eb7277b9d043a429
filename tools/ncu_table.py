"""Summarise an ncu --csv launch list: per-kernel time and DRAM bytes."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = None; data = {}; order = []
for r in rows:
    if r and r[0] == 'ID':
        hdr = r; continue
    if hdr is None or len(r) < len(hdr):
        continue
    d = dict(zip(hdr, r)); key = (int(d['ID']), d['Kernel Name'].split('(')[0].replace('void ', '')[:60])
    if key not in data:
        data[key] = {}; order.append(key)
    data[key][d['Metric Name']] = d['Metric Value']
tot = 0.0
for k in order:
    m = data[k]
    t = float(m.get('gpu__time_duration.sum', 0)) / 1e6
    tot += t
    rd = m.get('dram__bytes_read.sum'); wr = m.get('dram__bytes_write.sum'); hit = m.get('lts__t_sector_hit_rate.pct')
    extra = '' if rd is None else f" rd={float(rd)/1e9:7.2f}GB wr={float(wr)/1e9:6.2f}GB l2hit={hit}"
    print(f"{k[0]:4d} {t:9.3f} ms  {k[1]}{extra}")
print(f"total {tot:.3f} ms")
