"""Stall samples of an ncu source page per barrier-delimited SASS region.
    python tools/ncu_regions.py gpurun_out/prof_TAG"""
import csv
import sys

src = list(csv.reader(open(sys.argv[1] + ".source.csv")))
sh = src[1]
d = src[2:]
iS, iW = sh.index("Source"), sh.index("Warp Stall Sampling (All Samples)")
acc, start = 0, 0
for i, r in enumerate(d):
    acc += int(r[iW] or 0)
    s = r[iS]
    if "BAR.SYNC" in s or "EXIT" in s or i == len(d) - 1:
        if acc > 50:
            print(f"[{start:5d}-{i:5d}] samples={acc:6d}  ends with: {s.strip()[:50]}")
        acc, start = 0, i + 1
