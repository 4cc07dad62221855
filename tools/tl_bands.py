"""Band start/end times from a SAT_TIMELINE dump: how many bands are in flight
over time, and the implied output bandwidth (development tool)."""
import sys

bands = []
hdr = None
for line in open(sys.argv[1]):
    v = line.split()
    if v and v[0] == "launch":
        hdr = line.strip()
    elif v and v[0] == "band":
        bands.append((int(v[1]), int(v[2]), int(v[3])))
print(hdr)
t0 = min(b[1] for b in bands if b[1])
tend = max(b[2] for b in bands)
print(f"total {(tend - t0) / 1e3:.1f} us, {len(bands)} bands")
step = (tend - t0) / 20
for k in range(20):
    a, b = t0 + k * step, t0 + (k + 1) * step
    active = sum(1 for _, s, e in bands if s < b and e > a)
    done = sum(1 for _, s, e in bands if e <= b)
    print(f"  {a / 1e3 - t0 / 1e3:7.1f}-{b / 1e3 - t0 / 1e3:7.1f} us: active {active:4d}  done {done:4d}")
durs = sorted((e - s) / 1e3 for _, s, e in bands)
print(f"band duration (us): min {durs[0]:.1f} p50 {durs[len(durs)//2]:.1f} max {durs[-1]:.1f}")
for i in list(range(0, len(bands), max(1, len(bands) // 16))) + [len(bands) - 1]:
    g, s, e = bands[i]
    print(f"  band {g:5d}: start {(s - t0) / 1e3:7.1f}  end {(e - t0) / 1e3:7.1f}")
