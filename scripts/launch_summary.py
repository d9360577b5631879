"""Per-kernel share of an `ncu --metrics gpu__time_duration.sum --csv` launch list (cold-cache, serialised)."""
import csv
import re
import sys
from collections import defaultdict

rows = [r for r in csv.reader(l for l in open(sys.argv[1]) if not l.startswith("=="))]
h = rows[0]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
tot, cnt = defaultdict(float), defaultdict(int)
scale = {"ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "nsecond": 1e-6, "second": 1e3}
for r in rows[1:]:
    if len(r) <= max(ki, vi, ui):
        continue
    name = re.sub(r"\(.*", "", r[ki]).replace("void ", "").strip()
    tot[name] += float(r[vi].replace(",", "")) * scale.get(r[ui], 1e-6)
    cnt[name] += 1
T = sum(tot.values())
print(f"total {T:.3f} ms over {sum(cnt.values())} launches")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    print(f"{100 * v / T:6.2f}%  launches={cnt[k]:5d}  {v:9.3f} ms  {k}")
