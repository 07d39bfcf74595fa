"""Per-source-line instruction / stall shares from an ncu report
(`ncu -i REP --page source --csv --print-source cuda,sass` output on stdin)."""
import collections
import csv
import sys


def main():
    rows = list(csv.reader(sys.stdin))
    fname, hdr = None, None
    agg = collections.defaultdict(lambda: [0.0, 0.0, ""])
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < 8 or not r[0].isdigit():
            continue
        try:
            ss = float(r[4] or 0)
            ie = float(r[7] or 0)
        except ValueError:
            continue
        a = agg[(fname, int(r[0]))]
        a[0] += ie
        a[1] += ss
        a[2] = r[1][:80]
    ti = sum(v[0] for v in agg.values()) or 1
    ts = sum(v[1] for v in agg.values()) or 1
    top = int(sys.argv[1]) if len(sys.argv) > 1 else 30
    for (f, ln), v in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top]:
        print(f"{v[1] / ts * 100:5.1f}% stall {v[0] / ti * 100:5.1f}% inst  {f}:{ln}  {v[2]}")


if __name__ == "__main__":
    main()
