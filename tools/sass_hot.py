"""Hot SASS regions of an ncu report (ncu --page source --print-source sass CSV).

    python tools/sass_hot.py report.csv [N] [ex|stall]

Splits the instruction stream at branches into straight-line runs, ranks them
by warp-instructions executed (or stall samples), prints the top N with their
instructions (development tool)."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ia, isrc = hdr.index("Address"), hdr.index("Source")
iss = hdr.index("Warp Stall Sampling (All Samples)")
iex = hdr.index("Instructions Executed")
ins = []
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    ins.append((r[ia], r[isrc], int(float(r[iss] or 0)), int(float(r[iex] or 0))))
tot_ex = sum(i[3] for i in ins)
tot_s = sum(i[2] for i in ins)
blocks, cur = [], []
for i in ins:
    cur.append(i)
    if "BRA" in i[1] or "EXIT" in i[1] or "RET" in i[1]:
        blocks.append(cur)
        cur = []
if cur:
    blocks.append(cur)
N = int(sys.argv[2]) if len(sys.argv) > 2 else 12
key = sys.argv[3] if len(sys.argv) > 3 else "ex"
blocks.sort(key=lambda b: -(sum(i[3] for i in b) if key == "ex" else sum(i[2] for i in b)))
print(f"total warp-instr {tot_ex}  stall samples {tot_s}")
for b in blocks[:N]:
    ex = sum(i[3] for i in b)
    s = sum(i[2] for i in b)
    print(f"=== block @{b[0][0]} len {len(b)}  exec {ex} ({100*ex/tot_ex:.1f}%)  samples {s} ({100*s/tot_s:.1f}%)")
    for i in b:
        print(f"   {i[0]:>6} {i[3]:>10} {i[2]:>6}  {i[1]}")
