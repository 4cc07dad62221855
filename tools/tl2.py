"""SAT_TIMELINE dump -> per band (first band of each CTA): aggregate-sent,
V_up-landed and pass-B-done times at a few chunks, and the carry lag
(V_up - aggregate) (development tool)."""
import sys

launches = {}
cur = None
for line in open(sys.argv[1]):
    v = line.split()
    if not v:
        continue
    if v[0] == "launch":
        cur = line.split(" CL")[0]
        launches[cur] = (line.strip(), {})
    elif v[0] in ("cta", "agg", "vup"):
        b = int(v[1])
        d = launches[cur][1].setdefault(b, {})
        if v[0] == "cta":
            d["t0"], d["band"], d["pb"] = int(v[2]), int(v[3]), [int(x) for x in v[4:]]
        else:
            d[v[0]] = [int(x) for x in v[2:]]
for key, (hdr, ctas) in launches.items():
    print(hdr)
    T0 = min(d["t0"] for d in ctas.values() if d.get("t0"))
    rows = sorted(((d["band"] & 0xffffffff) + (d["band"] >> 32) * 100000, d) for d in ctas.values()
                  if d.get("pb") and d["pb"][0])
    nc = len(rows[0][1]["pb"])
    cols = sorted(set([0, 4, 8, 16, 24, nc - 1]) & set(range(nc)))
    print("  band  " + "".join(f"   c{c:<3d} agg/vup/pb      " for c in cols) + " lag(vup-agg) mean")
    step = max(1, len(rows) // 20)
    for i in list(range(0, len(rows), step)) + [len(rows) - 1]:
        band, d = rows[i]
        f = lambda x: (x - T0) / 1e3
        cells = []
        for c in cols:
            a, vv, p = d.get("agg", [0] * nc)[c], d.get("vup", [0] * nc)[c], d["pb"][c]
            cells.append(f"{f(a):6.1f}/{f(vv):6.1f}/{f(p):6.1f} ")
        lags = [(d["vup"][c] - d["agg"][c]) / 1e3 for c in range(nc) if d.get("vup") and d["vup"][c] and d["agg"][c]]
        print(f"  {band:5d} " + " ".join(cells) + f"  {sum(lags)/max(1,len(lags)):.2f}")
