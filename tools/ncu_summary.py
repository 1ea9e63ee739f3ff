"""Summarise the ncu captures of a round into profiles/.

    python tools/ncu_summary.py <round> [gpurun_out]

Reads gpurun_out/launches.csv (the --metrics gpu__time_duration.sum launch
list of `bench.py --steps 2 --warmup 3 --no-rows --no-e2e --no-cpu`) and
gpurun_out/prof_headline.ncu-rep (one --set full capture of the headline
kernel), writes profiles/ncu_launches_<round>.csv (copy), and
profiles/ncu_summary.json + profiles/ncu_<round>.md (kernel shares, DRAM bytes,
throughputs, occupancy, top stall reasons).
"""
import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launch_shares(path):
    """Kernel time shares from the first libds launch on (the warm-up and timed
    steps; input generation before it is excluded)."""
    rows = []
    with open(path) as fh:
        text = fh.read()
    start = text.find('"ID"')
    reader = csv.DictReader(io.StringIO(text[start:]))
    for r in reader:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        val = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "")
        ns = val * {"nsecond": 1, "ns": 1, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6,
                    "second": 1e9, "s": 1e9}.get(unit, 1)
        rows.append((r["Kernel Name"], ns))
    first = next((i for i, (k, _) in enumerate(rows) if "ds::" in k), 0)
    rows = rows[first:]
    tot = sum(ns for _, ns in rows)
    agg = {}
    for name, ns in rows:
        short = name.split("(")[0][:90]
        a = agg.setdefault(short, [0, 0.0])
        a[0] += 1
        a[1] += ns
    return tot, sorted(((k, c, ns) for k, (c, ns) in agg.items()), key=lambda x: -x[2])


def raw_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rd = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rd[0], rd[1], rd[2]
    return {h: (v, u) for h, u, v in zip(hdr, units, vals)}


def num(m, key):
    v, u = m.get(key, ("nan", ""))
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return None
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "ns": 1, "usecond": 1e3,
            "us": 1e3, "msecond": 1e6, "ms": 1e6}.get(u, 1)
    return x * mult


def main():
    rnd = sys.argv[1]
    src = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "gpurun_out")
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    summary = {"round": rnd}
    md = [f"# ncu summary, round {rnd}", ""]
    lc = os.path.join(src, "launches.csv")
    if os.path.exists(lc):
        shutil.copy(lc, os.path.join(prof, f"ncu_launches_{rnd}.csv"))
        tot, shares = launch_shares(lc)
        summary["launch_list"] = [{"kernel": k, "launches": c, "ns": ns, "share": ns / tot} for k, c, ns in shares]
        md += ["## Launch list (`ncu --metrics gpu__time_duration.sum`, cold-cache, serialised)", "",
               "Command: `bench.py --steps 2 --warmup 3 --no-rows --no-e2e --no-cpu` (C5, 1 GPU); "
               "launches from the first libds kernel on (warm-up + timed steps: restore copy, L2-flush "
               "read, compaction, count gather, offsets).", "",
               "| kernel | launches | total ms | share |", "|---|---|---|---|"]
        for k, c, ns in shares[:12]:
            md.append(f"| `{k}` | {c} | {ns / 1e6:.3f} | {ns / tot:.1%} |")
        md.append("")
    rep = os.path.join(src, "prof_headline.ncu-rep")
    if os.path.exists(rep):
        m = raw_metrics(rep)
        rd = num(m, "dram__bytes_read.sum")
        wr = num(m, "dram__bytes_write.sum")
        dur = num(m, "gpu__time_duration.sum")
        keys = ["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
                "sm__warps_active.avg.pct_of_peak_sustained_active",
                "launch__registers_per_thread", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
                "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_write.sum",
                "smsp__inst_executed.sum", "launch__grid_size", "launch__block_size"]
        head = {"kernel": m.get("Kernel Name", ("?", ""))[0], "dram_bytes_read": rd, "dram_bytes_write": wr,
                "dram_bytes_per_launch": (rd or 0) + (wr or 0), "duration_ns": dur}
        for k in keys:
            head[k] = num(m, k)
        summary["headline"] = head
        md += ["## Headline kernel (`ncu --set full`, one launch of the C5 compaction)", "",
               f"- kernel: `{head['kernel'][:100]}`",
               f"- duration under ncu: {dur / 1e6:.3f} ms (serialised, cold cache)" if dur else "",
               f"- DRAM read {rd / 1e9:.3f} GB, write {wr / 1e9:.3f} GB, total {(rd + wr) / 1e9:.3f} GB"
               if rd and wr else "",
               f"- DRAM throughput {head['gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed']} % of peak "
               f"(ncu's own peak), warps active {head['sm__warps_active.avg.pct_of_peak_sustained_active']} %, "
               f"registers {head['launch__registers_per_thread']}, grid {head['launch__grid_size']} x "
               f"{head['launch__block_size']}", ""]
    with open(os.path.join(prof, "ncu_summary.json"), "w") as fh:
        json.dump(summary, fh, indent=1)
    with open(os.path.join(prof, f"ncu_{rnd}.md"), "w") as fh:
        fh.write("\n".join(x for x in md if x is not None) + "\n")
    print(json.dumps(summary.get("headline", {}), indent=1))


if __name__ == "__main__":
    main()
