"""Top SASS instructions by warp-stall samples from an ncu report
(`ncu -i REP --page source --csv --print-source sass` on stdin)."""
import csv
import sys


def main():
    rows = list(csv.reader(sys.stdin))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
    h = rows[hdr]
    ia, isrc, ist, iex = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), \
        h.index("Instructions Executed")
    body = [r for r in rows[hdr + 1:] if len(r) > ist and r[0].startswith("0x")]
    tot = sum(float(r[ist] or 0) for r in body) or 1
    top = int(sys.argv[1]) if len(sys.argv) > 1 else 30
    idx = sorted(range(len(body)), key=lambda k: -float(body[k][ist] or 0))[:top]
    for k in sorted(idx):
        r = body[k]
        print(f"{k:5d} {float(r[ist] or 0) / tot * 100:5.1f}%  ex={r[iex]:>9}  {r[isrc].strip()[:90]}")


if __name__ == "__main__":
    main()
