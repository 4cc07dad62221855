"""Leader timeline (SAT_TIMELINE build, one-wave images): per cluster and
chunk, when the cluster's aggregates were all sent (max over its CTAs), when
the leader started (gather complete), knew the prefix, and sent V_up, and when
the bands' offset warps saw V_up (development tool)."""
import sys

d = {}
hdr = None
for line in open(sys.argv[1]):
    v = line.split()
    if not v:
        continue
    if v[0] == "launch":
        hdr = line.strip()
        d = {}
        cl = int(line.split("CL=")[1].split()[0])
    elif v[0] in ("cta", "agg", "vup", "ls", "lt", "ld", "rounds"):
        b = int(v[1])
        e = d.setdefault(b, {})
        if v[0] == "cta":
            e["t0"], e["band"] = int(v[2]), int(v[3])
        elif v[0] == "rounds":
            e["rounds"] = v[2:]
        else:
            e[v[0]] = [int(x) for x in v[2:]]
print(hdr)
T0 = min(e["t0"] for e in d.values() if e.get("t0"))
f = lambda x: (x - T0) / 1e3 if x else float("nan")
byband = {e["band"] & 0xffffffff: e for e in d.values() if "agg" in e}
nclus = (max(byband) + 1) // cl
chunks = [int(c) for c in (sys.argv[2].split(",") if len(sys.argv) > 2 else "0,1,8,16")]
print(" clus  chunk  agg_max  lead_start  prefix  vup_sent  vup_seen(max)   [lookback time, queue] rounds/retries")
for k in list(range(0, nclus, max(1, nclus // 16))) + [nclus - 1]:
    bands = [byband.get(k * cl + r) for r in range(cl)]
    if any(b is None for b in bands):
        continue
    for c in chunks:
        lead = bands[c % cl]
        am = max(b["agg"][c] for b in bands)
        vs = max(b["vup"][c] for b in bands)
        ls, lt, ld = lead["ls"][c], lead["lt"][c], lead["ld"][c]
        rr = lead.get("rounds", ["?"] * (c + 1))[c]
        print(f" {k:4d} {c:5d}  {f(am):7.1f}  {f(ls):9.1f}  {f(lt):7.1f}  {f(ld):7.1f}  {f(vs):9.1f}      [{(lt-ls)/1e3:5.1f} {(ls-am)/1e3:5.1f}] {rr}")
