"""Hot SASS regions of the first kernel in an `ncu --page source --csv --print-source sass` dump:
runs of consecutive instructions with equal execution counts, by share of executed instructions."""
import csv
import sys

lines = open(sys.argv[1]).read().split("\n")
blocks, cur = [], []
for l in lines:
    if l.startswith('"Kernel Name"'):
        if cur:
            blocks.append(cur)
        cur = []
    else:
        cur.append(l)
blocks.append(cur)
rows = list(csv.reader(blocks[int(sys.argv[2]) if len(sys.argv) > 2 else 0]))
hdr = rows[0]
rows = [r for r in rows[1:] if len(r) == len(hdr)]
ie, isamp = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
tot = sum(int(r[ie]) for r in rows)
segs = []
for r in rows:
    n = int(r[ie])
    if segs and segs[-1][0] == n:
        segs[-1][1] += 1
        segs[-1][3] += int(r[isamp])
        segs[-1][4].append(r[1].strip())
    else:
        segs.append([n, 1, r[0], int(r[isamp]), [r[1].strip()]])
print("total inst", tot)
for s in sorted(segs, key=lambda s: -s[0] * s[1])[:int(sys.argv[3]) if len(sys.argv) > 3 else 12]:
    print(f"{s[0]:>10} x {s[1]:>3} = {s[0]*s[1]/tot:6.1%}  samples {s[3]:>6}  @{s[2][-5:]}  " + " | ".join(s[4][:8]))
