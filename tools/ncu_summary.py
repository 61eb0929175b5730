"""Summarize ncu output into profiles/ (committed evidence).

  python tools/ncu_summary.py --launches gpurun_out/launches.csv \
      --report gpurun_out/prof.ncu-rep --tag r1 [--cells 16,512]

Writes profiles/<tag>_launches.md (kernel share of the bench command's launch
list: cold-cache, serialised per-launch times), profiles/<tag>_kernels.md (key
counters and the top stall sites of each captured launch) and
profiles/traffic.json (DRAM bytes per launch of the bulk kernels, read by
bench.py for the roofline's "traffic" field).
"""
import argparse
import collections
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", "L2 atomic requests (ALU)"),
    ("lts__t_requests_srcunit_tex_op_atom_dot_cas.sum", "L2 atomic requests (CAS)"),
    ("lts__t_requests_op_atom.sum", "L2 atom requests (all)"),
    ("lts__t_requests_op_red.sum", "L2 red requests"),
    ("lts__t_requests_op_atom.sum.per_second", "L2 atom requests / s"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum", "L1 global atom requests (warp instructions)"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_atom.sum", "L1 global atom sectors (address replay = sectors / requests)"),
    ("smsp__inst_executed_op_global_atom.sum", "global atom instructions executed"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "global load sectors"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors (from SM)"),
    ("l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum", "local-memory store sectors"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "active threads per instruction (divergence)"),
    ("smsp__sass_branch_targets_threads_divergent.sum", "divergent branch targets"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sectors.avg.pct_of_peak_sustained_elapsed", "L2 sector throughput % of peak"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall: long scoreboard / issue"),
    ("smsp__average_warps_issue_stalled_sleeping_per_issue_active.ratio", "stall: sleeping (spin waits) / issue"),
    ("smsp__average_warps_issue_stalled_membar_per_issue_active.ratio", "stall: membar / issue"),
]


def launches(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[start]
    ki, mi, vi, ui = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    agg = collections.defaultdict(list)
    for r in rows[start + 1:]:
        if len(r) > vi and r[mi] == "gpu__time_duration.sum":
            v = float(r[vi].replace(",", ""))
            v *= {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}.get(r[ui], 1.0)
            agg[r[ki].split("(")[0].replace("void ", "").replace("<unnamed>::", "")].append(v)
    return agg


def ncu_csv(report, page, extra=()):
    out = subprocess.run(["ncu", "-i", report, "--page", page, "--csv", *extra], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--report")
    ap.add_argument("--tag", default="r1")
    ap.add_argument("--cells", default="")
    ap.add_argument("--command", default="python bench.py --steps 2 --warmup 3 --no-extras --no-cpu")
    ap.add_argument("--capture", default="-k regex:k_bulk ... tools/prof_cells.py",
                    help="the captured command, for the report header")
    ap.add_argument("--traffic", action="store_true", help="write profiles/traffic.json (bulk-kernel DRAM bytes)")
    a = ap.parse_args()
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    if a.launches:
        agg = launches(a.launches)
        tot = sum(sum(v) for v in agg.values())
        lines = [f"# Launch list ({a.tag})", "",
                 f"`ncu --metrics gpu__time_duration.sum --clock-control none -c 600 {a.command}`", "",
                 "Cold-cache, serialised per-launch times: compare SHARES, not absolutes.", "",
                 "| kernel | launches | total µs | mean µs | share |", "|---|---:|---:|---:|---:|"]
        for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
            lines.append(f"| `{k[:70]}` | {len(v)} | {sum(v):.1f} | {sum(v) / len(v):.2f} | {sum(v) / tot:.1%} |")
        # the kernels of the bench's timed step only (the list above also holds
        # the untimed warm-up gate, post-run drain / stats and the RMW count)
        timed = {k: v for k, v in agg.items() if k.startswith(("k_reset", "k_bulk_malloc", "k_big", "k_bulk_free"))}
        tt = sum(sum(v) for v in timed.values()) or 1.0
        lines += ["", "Kernels of the timed step only (reset, malloc, batch kernel, free):", "",
                  "| kernel | launches | total µs | mean µs | share of the step's kernels |", "|---|---:|---:|---:|---:|"]
        for k, v in sorted(timed.items(), key=lambda x: -sum(x[1])):
            lines.append(f"| `{k[:70]}` | {len(v)} | {sum(v):.1f} | {sum(v) / len(v):.2f} | {sum(v) / tt:.1%} |")
        open(os.path.join(prof, f"{a.tag}_launches.md"), "w").write("\n".join(lines) + "\n")
    if a.report:
        raw = ncu_csv(a.report, "raw")
        hdr, units = raw[0], raw[1]
        cells = [c for c in a.cells.split(",") if c]
        lines = [f"# Kernel captures ({a.tag})", "",
                 f"`ncu --set full --clock-control none --import-source on {a.capture} {a.cells}`",
                 "", "One launch per row group (after one warm-up round)" +
                 ("; cells in order: " + a.cells if a.cells else ""), ""]
        traffic = {}
        src = ncu_csv(a.report, "source", ["--print-source", "sass"])
        stalls = []
        cur = None
        for r in src:
            if r and r[0] == "Kernel Name":
                cur = []
                stalls.append((r[1], cur))
            elif r and r[0] == "Address":
                shdr = r
            elif cur is not None and r:
                cur.append(r)
        for n, r in enumerate(raw[2:]):
            name = r[hdr.index("Kernel Name")]
            short = name.split("(")[0].replace("void ", "").replace("<unnamed>::", "")
            cell = cells[n // 2] if len(cells) * 2 == len(raw) - 2 else str(n)
            lines += [f"## `{short}` ({'cell ' + cell + ' B' if cells else 'launch ' + cell})", "",
                      "| counter | value |", "|---|---:|"]
            for m, label in METRICS:
                if m in hdr:
                    lines.append(f"| {label} (`{m}`) | {r[hdr.index(m)]} {units[hdr.index(m)]} |")
            rd = float(r[hdr.index("dram__bytes_read.sum")].replace(",", ""))
            wr = float(r[hdr.index("dram__bytes_write.sum")].replace(",", ""))
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            tb = rd * scale.get(units[hdr.index("dram__bytes_read.sum")], 1) + \
                wr * scale.get(units[hdr.index("dram__bytes_write.sum")], 1)
            key = "k_bulk_malloc" if "malloc" in short else ("k_bulk_free" if "free" in short else short)
            traffic.setdefault(key, {})[cell] = tb
            lines.append("")
        # top stall sites per distinct kernel (ncu aggregates per kernel name;
        # the source page repeats a kernel once per captured launch: keep one)
        seen = set()
        for name, rows in stalls:
            if name in seen:
                continue
            seen.add(name)
            si = shdr.index("Warp Stall Sampling (All Samples)")
            tot = sum(int(x[si]) for x in rows) or 1
            top = sorted(range(len(rows)), key=lambda i: -int(rows[i][si]))[:6]
            full = name.replace("void ", "").replace("<unnamed>::", "").replace("(anonymous namespace)::", "")
            lines += [f"### Top stall sites: `{full[:140]}` (every captured launch of this kernel, aggregated)", "",
                      "| share | SASS (stalled instruction; its producer precedes it) |", "|---:|---|"]
            for i in top:
                ctx = " ⟵ ".join(rows[j][1].strip()[:60] for j in range(i, max(-1, i - 3), -1))
                lines.append(f"| {int(rows[i][si]) / tot:.1%} | `{ctx}` |")
            lines.append("")
        open(os.path.join(prof, f"{a.tag}_kernels.md"), "w").write("\n".join(lines) + "\n")
        if not a.traffic:
            return
        tj = {k: (sum(v.values()) / len(v)) for k, v in traffic.items()}
        json.dump({"note": f"DRAM read+write bytes per launch from {a.tag} ncu --set full (mean over captured cells "
                           f"{a.cells})", **tj, "per_cell": traffic}, open(os.path.join(prof, "traffic.json"), "w"),
                  indent=1)


if __name__ == "__main__":
    main()
