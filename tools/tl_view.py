"""Print an SpMV timeline dump (MSP_SPMV_TL_FILE) relative to its start, us.
Producer: loop start, split searched, stage free, TMA issued.  Worker 0:
saw full, searched, gathers issued, products done, walked, published."""
import sys
rows = [list(map(int, l.split())) for l in open(sys.argv[1]) if l.strip()]
b0 = min(r[2] for r in rows if r[2] > 0)
cta = int(sys.argv[2]) if len(sys.argv) > 2 else 0
print("tile | prod: start srch  free  issue | work: full  srch gath  prod  walk  pub")
for r in rows:
    if r[0] != cta:
        continue
    v = [(x - b0) / 1000 if x else float("nan") for x in r[2:]]
    iss, full, walked, pub, srch, prod, gath, psr, pfree, pst = v[:10]
    print(f"{r[1]:4d} | {pst:7.2f} {psr-pst:5.2f} {pfree-psr:5.2f} {iss-pfree:5.2f} | {full:7.2f} {srch-full:5.2f} {gath-srch:5.2f} {prod-gath:5.2f} {walked-prod:5.2f} {pub-walked:5.2f}")
