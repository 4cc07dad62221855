"""Summarise tools/ab.sh output: mean ms per (config, library)."""
import collections
import re
import sys

res = collections.defaultdict(list)
cur = None
cfgs = []
for l in open(sys.argv[1]):
    if l.startswith("=="):
        cur = l.split("/")[-1].split(" (rep")[0].replace("libsat_", "").replace(".so", "")
    m = re.match(r"pair=(\d) (\S+): ([\d.]+) ms", l)
    if m:
        c = m.group(1) + " " + m.group(2)
        if c not in cfgs:
            cfgs.append(c)
        res[(c, cur)].append(float(m.group(3)))
libs = []
for (c, l) in res:
    if l not in libs:
        libs.append(l)
for i, l in enumerate(libs):
    print(f"  [{i}] {l}")
print("%-22s" % "cfg" + "".join("%10s" % f"[{i}]" for i in range(len(libs))))
for c in cfgs:
    print("%-22s" % c + "".join("%10s" % ("%.4f" % (sum(res[(c, l)]) / len(res[(c, l)])) if res[(c, l)] else "-") for l in libs))
