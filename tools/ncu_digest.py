"""Digest of an ncu capture made by tools/ncu_one.sh: key metrics, stall
reasons, hottest SASS lines.   python tools/ncu_digest.py gpurun_out/prof_TAG [--sass N]"""
import csv
import sys

base = sys.argv[1]
nsass = int(sys.argv[3]) if len(sys.argv) > 3 and sys.argv[2] == "--sass" else 25
rows = list(csv.reader(open(base + ".details.csv")))
h = rows[0]
iS, iM, iU, iV = (h.index(x) for x in ("Section Name", "Metric Name", "Metric Unit", "Metric Value"))
keep = {"Duration", "DRAM Throughput", "Memory Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Compute (SM) Throughput",
        "Achieved Occupancy", "Registers Per Thread", "Issue Slots Busy", "No Eligible", "Warp Cycles Per Issued Instruction",
        "Executed Ipc Active", "Mem Busy", "Max Bandwidth", "L1/TEX Cache Throughput", "L2 Cache Throughput",
        "Eligible Warps Per Scheduler"}
for r in rows[1:]:
    if r[iM] in keep:
        print(f"{r[iM]:40s} {r[iV]:>12s} {r[iU]}")
raw = list(csv.reader(open(base + ".raw.csv")))
hh, vv = raw[0], raw[2]
st = []
for i, k in enumerate(hh):
    if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued"):
        try:
            st.append((float(vv[i].replace(",", "")), k.replace("smsp__pcsamp_warps_issue_stalled_", "")))
        except ValueError:
            pass
for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct"):
    if k in hh:
        print(f"{k:40s} {vv[hh.index(k)]:>12s} {raw[1][hh.index(k)]}")
print("stalls:", ", ".join(f"{k}={int(v)}" for v, k in sorted(st, reverse=True)[:8]))
src = list(csv.reader(open(base + ".source.csv")))
sh = src[1]
d = src[2:]
iSrc, iW, iE = sh.index("Source"), sh.index("Warp Stall Sampling (All Samples)"), sh.index("Instructions Executed")
tot = sum(int(r[iW] or 0) for r in d)
print("samples", tot)
for idx, r in sorted(enumerate(d), key=lambda x: -int(x[1][iW] or 0))[:nsass]:
    print(f"{idx:5d} {int(r[iW]):7d} {r[iE]:>9s}  {r[iSrc].strip()}")
