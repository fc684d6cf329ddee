"""Expand launches of an ncu --metrics CSV sorted by duration: 'ID us MB share'."""
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 14 and r[0] != "ID"]
per = {}
for r in rows:
    if "expand" in r[4]:
        v = float(r[14].replace(",", ""))
        per.setdefault(int(r[0]), {})[r[12]] = v
tot = sum(x.get("gpu__time_duration.sum", 0) for x in per.values()) or 1
for i, x in sorted(per.items(), key=lambda kv: -kv[1].get("gpu__time_duration.sum", 0)):
    t = x.get("gpu__time_duration.sum", 0)
    mb = (x.get("dram__bytes_read.sum", 0) + x.get("dram__bytes_write.sum", 0)) / 1e6
    print(f"{i} {t / 1e3:.1f} {mb:.1f} {t / tot:.3f}")
