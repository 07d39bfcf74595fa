# Digest an ncu report on the box (reports are too large to bring back):
#   bash tools/ncu_digest.sh REP.ncu-rep OUTPREFIX
rep=$1; out=$2
ncu -i "$rep" --page details --csv > "$out.details.csv" 2>/dev/null
ncu -i "$rep" --page raw --csv > "$out.raw.csv" 2>/dev/null
ncu -i "$rep" --page source --csv --print-source sass 2>/dev/null | python tools/ncu_sass_top.py 60 > "$out.sass_top.txt"
ncu -i "$rep" --page source --csv --print-source sass 2>/dev/null | gzip > "$out.sass.csv.gz"
rm -f "$rep"
