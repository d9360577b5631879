#!/usr/bin/env python
"""Blackwell-native instruction evidence for libsr.so's kernels (no GPU needed): per kernel function, the number of
SASS instructions of each family in `cuobjdump -sass` (B200_PROFILING.md: tcgen05.mma -> UTC*MMA, tcgen05.ld/st ->
LDTM/STTM, TMA -> UTMALDG/UTMASTG/UBLKCP, legacy mma.sync -> HMMA).  Writes a markdown table (stdout) and JSON
(--json PATH)."""
import argparse
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FAMILIES = {
    "UTC*MMA (tcgen05.mma)": re.compile(r"\bUTC\w*MMA\b"),
    "LDTM (tcgen05.ld)": re.compile(r"\bLDTM\b"),
    "STTM (tcgen05.st)": re.compile(r"\bSTTM\b"),
    "UTMALDG (TMA load)": re.compile(r"\bUTMALDG\b"),
    "UTMASTG (TMA store)": re.compile(r"\bUTMASTG\b"),
    "UBLKCP (bulk copy)": re.compile(r"\bUBLKCP\b"),
    "HMMA (legacy mma.sync)": re.compile(r"\bHMMA\b"),
}


def demangle(names):
    try:
        out = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.splitlines()
        return out if len(out) == len(names) else names
    except OSError:
        return names


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lib", default=os.path.join(ROOT, "paper_conf_sigcomm_kimjyyh20_b200", "libsr.so"))
    ap.add_argument("--json", default=None)
    args = ap.parse_args()
    sass = subprocess.run(["cuobjdump", "-sass", args.lib], capture_output=True, text=True, check=True).stdout
    funcs = {}
    cur = None
    for ln in sass.splitlines():
        m = re.match(r"\s*Function : (\S+)", ln)
        if m:
            cur = m.group(1)
            funcs[cur] = {k: 0 for k in FAMILIES}
            continue
        if cur is None:
            continue
        for k, rx in FAMILIES.items():
            if rx.search(ln):
                funcs[cur][k] += 1
    names = list(funcs)
    pretty = demangle(names)
    rows = []
    for raw, nice in zip(names, pretty):
        c = funcs[raw]
        if not any(c.values()) and not raw.startswith("_Z"):
            continue
        short = re.sub(r"\(.*", "", nice).replace("sr::", "")
        rows.append((short, c))
    rows.sort(key=lambda r: (-r[1]["UTC*MMA (tcgen05.mma)"], r[0]))
    hdr = "| kernel | " + " | ".join(FAMILIES) + " |"
    print(hdr)
    print("|" + "---|" * (len(FAMILIES) + 1))
    for name, c in rows:
        print(f"| `{name}` | " + " | ".join(str(c[k]) for k in FAMILIES) + " |")
    if args.json:
        with open(args.json, "w") as f:
            json.dump({n: c for n, c in rows}, f, indent=1)
    return 0


if __name__ == "__main__":
    sys.exit(main())
