"""Per-kernel table of an ncu launch list (gpu__time_duration + dram bytes) for the last step."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
first = sys.argv[2] if len(sys.argv) > 2 else "lazy_reset"
hdr = None
per = {}
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        k = (int(d["ID"]), d["Kernel Name"].split("(")[0][-40:])
        per.setdefault(k, {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
items = sorted(per.items())
idx = [i for i, (k, v) in enumerate(items) if first in k[1]]
tot = 0.0
for k, v in items[idx[-1] if idx else 0:]:
    if "k_mb_" in k[1]:
        break
    t = v.get("gpu__time_duration.sum", 0) / 1e3
    tot += t
    print(f"{k[1]:42s} {t:9.1f} us  rd {v.get('dram__bytes_read.sum', 0) / 1e9:7.2f} GB  wr "
          f"{v.get('dram__bytes_write.sum', 0) / 1e9:7.2f} GB")
print(f"{'total':42s} {tot:9.1f} us")
