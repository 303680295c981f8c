"""Top SASS instructions by warp-stall samples from `ncu --page source --csv --print-source sass`."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
idx = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
tot = sum(int(r[idx['Warp Stall Sampling (All Samples)']] or 0) for r in data if len(r) == len(hdr))
top = sorted((r for r in data if len(r) == len(hdr)), key=lambda r: -int(r[idx['Warp Stall Sampling (All Samples)']] or 0))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
stall_cols = [h for h in hdr if h.startswith('stall_')]
for r in top[:n]:
    s = int(r[idx['Warp Stall Sampling (All Samples)']] or 0)
    stalls = sorted(((int(r[idx[c]] or 0), c[6:]) for c in stall_cols), reverse=True)[:2]
    print(f"{100*s/tot:5.1f}% {r[idx['Address']][-5:]} {r[idx['Source']].strip()[:60]:60s} {stalls}")
print("total samples", tot, "instructions", len(data))
