"""Summarise ncu captures brought back in gpurun_out/ into committed files.

    python profiles/summarize.py launches <launches.csv> <out.txt>
    python profiles/summarize.py full <report.ncu-rep> <out.txt> [--traffic-key app:kernel]

`launches`: per-kernel launch counts, total/mean device time and share of the
captured time (ncu's cold-cache, serialised per-launch times — compare shares).
`full`: the metrics the roofline uses (duration, DRAM bytes read/written,
DRAM throughput %, registers, occupancy); with --traffic-key the mean DRAM
bytes per launch is merged into profiles/ncu_traffic.json for bench.py.
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))


def launches(path, out):
    rows = []
    with open(path) as f:
        lines = [l for l in f if not l.startswith("==")]
    r = csv.DictReader(io.StringIO("".join(lines)))
    for row in r:
        if row.get("Metric Name") == "gpu__time_duration.sum":
            v = float(row["Metric Value"].replace(",", ""))
            unit = row.get("Metric Unit", "")
            scale = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "us": 1.0, "ns": 1e-3, "ms": 1e3}.get(unit, 1.0)
            rows.append((row["Kernel Name"], v * scale))
    agg = collections.OrderedDict()
    for name, us in rows:
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += us
    tot = sum(a[1] for a in agg.values()) or 1.0
    with open(out, "w") as f:
        f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none launch list: {os.path.basename(path)}\n")
        f.write(f"# {len(rows)} launches, {tot:.1f} us total (cold-cache, serialised)\n")
        f.write(f"{'launches':>8} {'total_us':>12} {'mean_us':>10} {'share':>7}  kernel\n")
        for name, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            f.write(f"{n:8d} {us:12.1f} {us / n:10.2f} {us / tot:7.1%}  {name[:110]}\n")
    print(open(out).read())


METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size", "launch__block_size",
           "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active",
           "lts__t_bytes.sum", "launch__shared_mem_per_block_dynamic"]


def full(rep, out, key=None):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m in METRICS:
            if m in hdr:
                d[m] = (r[hdr.index(m)], units[hdr.index(m)])
        res.append(d)
    with open(out, "w") as f:
        f.write(f"# ncu --set full --clock-control none: {os.path.basename(rep)}\n")
        for d in res:
            f.write(f"kernel: {d['kernel'][:140]}\n")
            for m in METRICS:
                if m in d:
                    f.write(f"  {m:70s} {d[m][0]:>14} {d[m][1]}\n")
    print(open(out).read())
    if key:
        def gb(v):
            x, u = v
            x = float(x.replace(",", ""))
            return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)
        traf = [gb(d["dram__bytes_read.sum"]) + gb(d["dram__bytes_write.sum"]) for d in res]
        path = os.path.join(HERE, "ncu_traffic.json")
        data = json.load(open(path)) if os.path.exists(path) else {}
        data[key] = max(traf)
        json.dump(data, open(path, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    mode, src, dst = sys.argv[1:4]
    key = sys.argv[sys.argv.index("--traffic-key") + 1] if "--traffic-key" in sys.argv else None
    launches(src, dst) if mode == "launches" else full(src, dst, key)
