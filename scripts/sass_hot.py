"""Top SASS lines by warp-stall samples from `ncu --page source --csv --print-source sass`."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
ia, isrc = hdr.index("Address"), hdr.index("Source")
iss, iex = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
tot = sum(float(r[iss] or 0) for r in data) or 1.0
print(f"# hottest SASS lines ({rows[0][0] if rows[0] else ''}: {rows[0][1][:90] if len(rows[0]) > 1 else ''})\n")
print(f"total warp-stall samples: {tot:.0f}\n")
print("| samples | share | executed | SASS |\n|---|---|---|---|")
for r in sorted(data, key=lambda r: -float(r[iss] or 0))[:25]:
    print(f"| {float(r[iss] or 0):.0f} | {100 * float(r[iss] or 0) / tot:.1f}% | {r[iex]} | `{r[isrc].strip()[:70]}` |")
