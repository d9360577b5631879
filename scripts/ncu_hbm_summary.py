"""Per-launch duration and DRAM bytes (read + write) from `ncu --metrics gpu__time_duration.sum,dram__bytes_*
--csv` captures: one line per capture file (mean over its launches), GB/s = DRAM bytes / duration."""
import collections
import csv
import os
import re
import sys

SC = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "nsecond": 1e-9, "us": 1e-6, "usecond": 1e-6,
      "ms": 1e-3, "msecond": 1e-3}
for path in sys.argv[1:]:
    try:
        rows = [r for r in csv.reader(ln for ln in open(path) if not ln.startswith("=="))]
    except OSError:
        continue
    if not rows:
        continue
    h = rows[0]
    ki, mi, vi, ui, ii = (h.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit", "ID"))
    per = collections.defaultdict(dict)
    name = ""
    for r in rows[1:]:
        if len(r) <= vi:
            continue
        per[r[ii]][r[mi]] = float(r[vi].replace(",", "")) * SC.get(r[ui], 1.0)
        name = re.sub(r"\(.*", "", r[ki]).replace("void ", "")
    if not per:
        continue
    n = len(per)
    t = sum(m["gpu__time_duration.sum"] for m in per.values()) / n
    rd = sum(m["dram__bytes_read.sum"] for m in per.values()) / n
    wr = sum(m["dram__bytes_write.sum"] for m in per.values()) / n
    tag = os.path.basename(path).replace("r02_ncu_hbm_", "").replace(".csv", "")
    print(f"{tag:12s} {name[:44]:44s} launches={n} dur={t * 1e6:9.2f} us  dram read={rd / 1e6:9.3f} MB "
          f"write={wr / 1e6:9.3f} MB  -> {(rd + wr) / t / 1e9:8.1f} GB/s")
