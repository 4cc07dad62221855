"""Summarise a SAT_TIMELINE dump (development tool): for the last launch of each
shape, the pass-B completion time of every chunk of each CTA's first band."""
import sys

launches = {}
cur = None
for line in open(sys.argv[1]):
    if line.startswith("launch"):
        cur = line.split(" CL")[0]
        launches[cur] = (line.strip(), [])
    elif line.startswith("cta"):
        v = line.split()
        launches[cur][1].append((int(v[1]), int(v[2]), int(v[3]), [int(x) for x in v[4:]]))
for key, (hdr, ctas) in launches.items():
    t0 = min(c[1] for c in ctas)
    print(hdr)
    st = sorted((c[1] - t0) / 1e3 for c in ctas if c[1])
    print("  CTA start (us): min %.1f p50 %.1f p90 %.1f max %.1f  (n=%d)" % (st[0], st[len(st)//2], st[int(len(st)*0.9)], st[-1], len(st)))
    rows = sorted(((c[2] & 0xffffffff) + (c[2] >> 32) * 100000, c) for c in ctas if c[3] and c[3][0])
    nc = len(rows[0][1][3])
    cols = sorted(set([0, 1, 2, 4, 8, 16, 32, 48, nc - 1]) & set(range(nc)))
    print("  band   " + " ".join(f"c{c:<6d}" for c in cols) + "  pace(us/chunk) first->last")
    step = max(1, len(rows) // 24)
    for i in list(range(0, len(rows), step)) + [len(rows) - 1]:
        band, c = rows[i]
        ts = [(x - t0) / 1e3 for x in c[3]]
        pace = (ts[-1] - ts[0]) / max(1, len(ts) - 1)
        print(f"  {band:6d} " + " ".join(f"{ts[k]:7.1f}" for k in cols) + f"  {pace:.2f}")
