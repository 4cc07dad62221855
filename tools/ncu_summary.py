"""Summarise ncu captures into profiles/ (tracked).

    python tools/ncu_summary.py ROUND REP [REP ...] [--launches CSV]

For every `ncu --set full` report: duration, DRAM bytes read/written, DRAM
throughput, issue/occupancy figures and the top warp-stall reasons.  Writes
profiles/<ROUND>_ncu.md (human) and merges per-workload DRAM bytes into
profiles/ncu_summary.json (read by bench.py for roofline.traffic).
"""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROFILES = os.environ.get("NCU_SUMMARY_DIR") or os.path.join(ROOT, "profiles")
KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct_peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_pct_peak"),
    ("lts__t_bytes.sum", "l2_bytes"),
    ("smsp__inst_executed.sum", "warp_inst"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy_pct"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_active_pct"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "lsu_pct"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__shared_mem_per_block_dynamic", "smem_dyn"),
]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
        "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}
WORKLOAD_OF = {  # prof_one args -> bench workload name
    "p0_16384x16384x1": "sweep-16384sq-8u32s",
    "p1_16384x16384x1": "sweep-16384sq-32f32f",
    "p0_8192x8192x1": "sweep-8192sq-8u32s",
    "p0_1080x1920x1024": "batch-1024x1080x1920-8u32s",
    "p1_65536x65536x1": "huge-65536sq-32f32f",
    "p2_16384x16384x1": "64f-16384sq",
    "p5_16384x16384x1": "sq-16384sq-8u",
    "p6_16384x16384x1": "hist4-16384sq-8u",
    "p1_8192x8192x1": "sweep-8192sq-32f32f",
    "p2_4096x65536x1": "64f-4096x65536",
    "p3_16384x16384x1": "8u32f-16384sq",
    "p1_4096x65536x1": "32f-4096x65536",
}
IN_B = {0: 1, 1: 4, 2: 8, 3: 1, 4: 4, 5: 1, 6: 1}
OUT_B = {0: 4, 1: 4, 2: 8, 3: 4, 4: 4, 5: 8, 6: 16}


def raw(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True,
                                  stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for k, name in KEYS:
        if k in hdr:
            i = hdr.index(k)
            try:
                v = float(vals[i].replace(",", ""))
            except ValueError:
                continue
            d[name] = v * UNIT.get(units[i], 1.0)
    stalls = {}
    for i, h in enumerate(hdr):
        m = re.match(r"smsp__average_warps_issue_stalled_(\w+)_per_issue_active\.ratio$", h)
        if m:
            try:
                stalls[m.group(1)] = float(vals[i])
            except ValueError:
                pass
    d["top_stalls"] = sorted(stalls.items(), key=lambda kv: -kv[1])[:6]
    d["kernel"] = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
    return d


def main():
    args = sys.argv[1:]
    rnd = args.pop(0)
    launches = None
    if "--launches" in args:
        i = args.index("--launches")
        launches = args[i + 1]
        del args[i:i + 2]
    summary_path = os.path.join(PROFILES, "ncu_summary.json")
    summary = json.load(open(summary_path)) if os.path.exists(summary_path) else {}
    lines = [f"# ncu summary, {rnd}", "",
             "Captured with `ncu --set full --clock-control none --import-source on -k regex:sat_tile "
             "-s 2 -c 1` on one B200 (tools/prof_one.py: 3 launches, the 3rd profiled).  ncu times are "
             "cold-cache, serialised replays: compare shares, not absolutes.", "",
             "| config | kernel | duration us | DRAM read MB | DRAM write MB | alg. bytes MB | "
             "traffic/alg | DRAM % peak | issue % | occupancy % | regs | top stalls (cycles/issue) |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for rep in args:
        tag = re.search(r"(p\d_\d+x\d+x\d+)", rep).group(1)
        pair, shape = int(tag[1]), tag[3:]
        H, W, N = (int(v) for v in shape.split("x"))
        d = raw(rep)
        alg = H * W * N * (IN_B[pair] + OUT_B[pair])
        traffic = d.get("dram_read", 0) + d.get("dram_write", 0)
        st = ", ".join(f"{k} {v:.1f}" for k, v in d["top_stalls"][:4])
        kern = re.sub(r"\(.*", "", d["kernel"])
        lines.append(f"| {tag} | {kern} | {d.get('duration', 0) * 1e6:.1f} | "
                     f"{d.get('dram_read', 0) / 1e6:.1f} | {d.get('dram_write', 0) / 1e6:.1f} | "
                     f"{alg / 1e6:.1f} | {traffic / alg:.3f} | {d.get('dram_pct_peak', 0):.1f} | "
                     f"{d.get('issue_active_pct', 0):.1f} | {d.get('occupancy_pct', 0):.1f} | "
                     f"{d.get('regs', 0):.0f} | {st} |")
        wl = WORKLOAD_OF.get(tag)
        if wl:
            summary[wl] = {"dram_bytes_per_launch": traffic, "algorithmic_bytes": alg,
                           "ncu_duration_us": d.get("duration", 0) * 1e6, "round": rnd,
                           "report": os.path.basename(rep)}
    if launches:
        lines += ["", f"## Launch list (`{os.path.basename(launches)}`)", ""]
        tot = {}
        with open(launches) as f:
            text = f.read()
        start = text.find('"ID"')
        rows = list(csv.DictReader(io.StringIO(text[start:])))
        for r in rows:
            if r.get("Metric Name") != "gpu__time_duration.sum":
                continue
            k = re.sub(r"\(.*", "", r["Kernel Name"])
            v = float(r["Metric Value"].replace(",", "")) * UNIT.get(r["Metric Unit"], 1.0)
            tot.setdefault(k, [0, 0.0])
            tot[k][0] += 1
            tot[k][1] += v
        allt = sum(v[1] for v in tot.values())
        lines += ["| kernel | launches | total ms | share |", "|---|---|---|---|"]
        for k, (n, t) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
            lines.append(f"| {k} | {n} | {t * 1e3:.3f} | {t / allt:.1%} |")
    os.makedirs(PROFILES, exist_ok=True)
    open(os.path.join(PROFILES, f"{rnd}_ncu.md"), "w").write("\n".join(lines) + "\n")
    json.dump(summary, open(summary_path, "w"), indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
