"""Summarise an `ncu --csv --metrics ...` launch list: one line per launch
(kernel, duration us, DRAM read/write MB).  Usage: python tools/ncu_csv.py FILE [LAST_N]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
last = int(sys.argv[2]) if len(sys.argv) > 2 else 0
hdr = None
agg = collections.OrderedDict()
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr):
        continue
    d = dict(zip(hdr, r))
    agg.setdefault((d["ID"], d["Kernel Name"]), {})[d["Metric Name"]] = d["Metric Value"].replace(",", "")
items = list(agg.items())[-last:] if last else list(agg.items())
for (i, k), v in items:
    t = float(v.get("gpu__time_duration.sum", 0)) / 1e3
    rd = float(v.get("dram__bytes_read.sum", 0)) / 1e6
    wr = float(v.get("dram__bytes_write.sum", 0)) / 1e6
    print(f"{i:>4} {k.split('(')[0][:44]:44s} {t:9.1f} us  rd {rd:8.1f} MB  wr {wr:8.1f} MB  {(rd + wr) / max(t, 1e-9) / 1e3:6.2f} TB/s")
