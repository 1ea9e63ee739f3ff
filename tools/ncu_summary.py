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


def role_samples(rep, src_file):
    """Warp-state samples per role of the irregular kernel, from the cuda,sass
    source view (-lineinfo + --import-source): lines of ds_irregular.cu are
    attributed to the function / role section that contains them, by the
    section markers in the source; inlined helpers from other files count as
    'helpers'.  'look-back' = the decoupled look-back's poll loop (the
    flag-spin of SURVEY 8(d))."""
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    with open(src_file) as fh:
        lines = fh.read().split("\n")

    def find(pat):
        return next((i + 1 for i, x in enumerate(lines) if pat in x), None)
    marks = sorted((v, k) for k, v in {
        "look-back": find("uint64_t lookback("), "look-back (local chain)": find("uint64_t lookback_window("),
        "storers (STG helper)": find("void store_segment("), "storers (re-phase)": find("void rephase("),
        "end-aware waits": find("bool mbar_wait_or_end("),
        "rankers (keep bits)": find("uint32_t keep_bits4("),
        "kernel setup": find("__global__ void __launch_bounds__"),
        "producer": find("---- producer"), "rankers": find("---- ranker warps"),
        "resolvers": find("---- resolver warps"), "storers": find("---- storer warps"),
        "host": find("struct LaunchCache")}.items() if v)
    roles, cur_file, col = {}, None, None
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] in ("File Path", "File Name"):
            cur_file = r[1]
            continue
        if r[0] == "Line No":
            col = r.index("Warp Stall Sampling (All Samples)")
            continue
        if col is None or not r[0].isdigit():
            continue
        try:
            smp = int(r[col])
        except ValueError:
            continue
        if cur_file and os.path.basename(cur_file) == os.path.basename(src_file):
            ln = int(r[0])
            role = "other"
            for start, name in marks:
                if ln >= start:
                    role = name
        else:
            role = "helpers (" + os.path.basename(cur_file or "?") + ")"
        roles[role] = roles.get(role, 0) + smp
    return roles


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
        if os.path.exists(rep):
            roles = role_samples(rep, os.path.join(ROOT, "paper_conf_icpp_gomez_lunacshg15_b200", "csrc",
                                                   "ds_irregular.cu"))
            tot = sum(roles.values())
            if tot:
                summary["warp_samples_by_role"] = roles
                summary["flag_spin_fraction"] = roles.get("look-back", 0) / tot
                md += ["## Warp-state samples by role (source view, all warps of the headline kernel)", "",
                       "| role | samples | share |", "|---|---|---|"]
                for k, v in sorted(roles.items(), key=lambda kv: -kv[1]):
                    md.append(f"| {k} | {v} | {v / tot:.1%} |")
                md += ["", f"Flag-spin fraction (samples in the look-back poll loop / all samples): "
                       f"{summary['flag_spin_fraction']:.1%}.  The look-back runs on dedicated resolver "
                       "warps, so these samples are parked pollers, not stalled data movers; the "
                       "rankers' share is the busy fraction of the ranking step.", ""]
        ld_sec = num(m, "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum")
        ld_req = num(m, "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")
        st_sec = num(m, "l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum")
        st_req = num(m, "l1tex__t_requests_pipe_lsu_mem_global_op_st.sum")
        if ld_req and st_req:
            summary["lsu_sectors_per_request"] = {"ld": ld_sec / ld_req, "st": st_sec / st_req}
            md += [f"LSU sectors/request: loads {ld_sec / ld_req:.1f} (the status polls: 32 statuses 64 B apart "
                   f"per warp load), stores {st_sec / st_req:.1f} (status words and the <= 6 scalar head/tail "
                   "words per tile).  The tile data moves through TMA bulk copies, not the LSU.", ""]
    with open(os.path.join(prof, "ncu_summary.json"), "w") as fh:
        json.dump(summary, fh, indent=1)
    with open(os.path.join(prof, f"ncu_{rnd}.md"), "w") as fh:
        fh.write("\n".join(x for x in md if x is not None) + "\n")
    print(json.dumps(summary.get("headline", {}), indent=1))


if __name__ == "__main__":
    main()
