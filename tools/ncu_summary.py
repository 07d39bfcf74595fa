"""Summarise an `ncu --page raw --csv` export into a small JSON (the numbers
bench.py's roofline.traffic and DESIGN.md cite).

    python tools/ncu_summary.py RAW.csv OUT.json "source description" [kernel-regex]
"""
import csv
import json
import re
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_shared_mem",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "us": 1, "usecond": 1, "msecond": 1e3,
         "ms": 1e3, "nsecond": 1e-3}


def main():
    src, out, desc = sys.argv[1], sys.argv[2], sys.argv[3]
    pat = re.compile(sys.argv[4]) if len(sys.argv) > 4 else None
    rows = list(csv.reader(open(src)))
    hdr, units = rows[0], rows[1]
    launches = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        if pat and not pat.search(d.get("Kernel Name", "")):
            continue
        e = {"kernel": d.get("Kernel Name", "")[:160]}
        for k in KEYS:
            if k in d and d[k] not in ("", None):
                u = units[hdr.index(k)]
                try:
                    v = float(d[k].replace(",", ""))
                except ValueError:
                    continue
                e[k] = v * SCALE.get(u, 1) if u in SCALE else v
                e[k + ".unit"] = "byte" if u.endswith("byte") else ("us" if u in SCALE and "s" in u else u)
        st = {h: float(v.replace(",", "")) for h, v in d.items()
              if h.startswith("smsp__pcsamp_warps_issue_stalled") and not h.endswith("not_issued") and v}
        tot = sum(st.values()) or 1
        e["stall_shares"] = {h.replace("smsp__pcsamp_warps_issue_stalled_", ""): round(v / tot, 4)
                             for h, v in sorted(st.items(), key=lambda kv: -kv[1])[:10]}
        launches.append(e)
    res = {"source": desc, "launches": launches}
    if launches:
        b = [x.get("dram__bytes_read.sum", 0) + x.get("dram__bytes_write.sum", 0) for x in launches]
        res["dram_bytes_per_launch"] = sum(b) / len(b)
        res["duration_us"] = sum(x.get("gpu__time_duration.sum", 0) for x in launches) / len(launches)
    json.dump(res, open(out, "w"), indent=1)
    print(json.dumps({k: v for k, v in res.items() if k != "launches"}))


if __name__ == "__main__":
    main()
