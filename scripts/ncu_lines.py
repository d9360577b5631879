"""Per-source-line warp-stall samples of an ncu report (`--page source --print-source cuda,sass`): the lines
(file:line, over every inlined header) with the most samples and their top stall reasons."""
import csv
import subprocess
import sys


def main(path, top=40):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    fpath, h, agg = "?", None, {}
    for r in csv.reader(out.splitlines()):
        if not r:
            continue
        if r[0] == "File Path":
            fpath = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            h = r
            continue
        if h is None or r[0] == "" or r[0] == "Function Name":
            continue
        d = dict(zip(h[:2], r[:2]))
        vals = r[4:]
        names = h[4:]
        row = dict(zip(names, vals))
        try:
            s = int(row.get("Warp Stall Sampling (All Samples)", "0") or 0)
        except ValueError:
            continue
        if s <= 0:
            continue
        st = {k: int(v) for k, v in row.items() if k.startswith("stall_") and "(Not" not in k and v.isdigit() and v != "0"}
        agg[(fpath, int(d["Line No"]))] = (s, r[1].strip()[:80], st)
    tot = sum(v[0] for v in agg.values())
    print(f"total samples {tot}")
    for (f, l), (s, src, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        t3 = ", ".join(f"{k[6:]}={v}" for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:3])
        print(f"{s:6d} {100 * s / tot:5.1f}%  {f}:{l:<4d} {src:80s} | {t3}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)
