"""Instruction and stall totals per CUDA source line from `ncu --page source --csv --print-source sass`
(the SASS rows carry the source line they were compiled from when built with -lineinfo)."""
import csv, sys, collections, re
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
idx = {h: i for i, h in enumerate(hdr)}
data = [r for r in rows[2:] if len(r) == len(hdr)]
def f(r, k):
    try:
        return float(r[idx[k]] or 0)
    except (ValueError, KeyError):
        return 0.0
tot_i = sum(f(r, 'Instructions Executed') for r in data)
tot_s = sum(f(r, 'Warp Stall Sampling (All Samples)') for r in data)
ops = collections.Counter(); st = collections.Counter()
for r in data:
    src = r[idx['Source']].strip()
    op = re.sub(r'^@!?U?P\w+\s+', '', src).split()[0] if src else '?'
    ops[op] += f(r, 'Instructions Executed'); st[op] += f(r, 'Warp Stall Sampling (All Samples)')
print(f"total warp instructions {tot_i:.3e}, stall samples {tot_s:.0f}")
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for op, c in ops.most_common(n):
    print(f"{op:24s} {100*c/tot_i:5.1f}% inst  {100*st[op]/max(tot_s,1):5.1f}% stall")
