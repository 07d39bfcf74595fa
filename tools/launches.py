"""Summarise an `ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum --csv` launch list: one line per launch (ms, GB read,
GB written), optionally filtered by a kernel-name substring.

    python tools/launches.py gpurun_out/x/launches.csv [substring]"""
import collections
import csv
import sys


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    flt = sys.argv[2] if len(sys.argv) > 2 else ""
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    agg = collections.OrderedDict()
    for r in rows[start + 1:]:
        if len(r) < len(hdr):
            continue
        key = (int(r[0]), r[ki])
        agg.setdefault(key, {})[r[mi]] = float(r[vi].replace(",", ""))
    tot = 0.0
    for (i, k), d in agg.items():
        if flt not in k:
            continue
        ms = d.get("gpu__time_duration.sum", 0) / 1e6
        tot += ms
        print(f"{i:4d} {ms:9.3f} ms  rd {d.get('dram__bytes_read.sum', 0) / 1e9:8.2f} GB  "
              f"wr {d.get('dram__bytes_write.sum', 0) / 1e9:7.2f} GB  {k[:90]}")
    print(f"total {tot:.3f} ms")


if __name__ == "__main__":
    main()
