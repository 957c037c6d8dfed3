"""Summarise ncu captures into profiles/ (tracked): key metrics of a --set full report and
the per-kernel shares of a launch list.  Usage:
  python scripts/summarize_ncu.py full <report.ncu-rep> <out-prefix> <computed_cell_dims>
  python scripts/summarize_ncu.py launches <launches.csv> <out.txt>
"""
import collections
import csv
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "launch__registers_per_thread", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "smsp__inst_executed.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed"]


def full(rep, prefix, cells):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units, vals = rows[0], rows[1], rows[2]
    out = {"report": rep, "kernel": vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else None}
    for h, u, v in zip(hdr, units, vals):
        if h in KEYS or ("issue_stalled" in h and "per_issue_active" in h):
            try:
                out[h] = (float(v.replace(",", "")), u)
            except ValueError:
                pass
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout.splitlines()
    srows = list(csv.reader(src))
    sh = srows[1]
    ix = {h: i for i, h in enumerate(sh)}
    ops = collections.Counter()
    tot = 0
    for r in srows[2:]:
        if len(r) < len(sh):
            continue
        nexe = int(r[ix["Instructions Executed"]] or 0)
        tok = r[ix["Source"]].strip().split()
        if not tok:
            continue
        o = tok[1] if tok[0].startswith("@") else tok[0]
        ops[o.split(".")[0]] += nexe
        tot += nexe
    cells = float(cells)
    out["thread_instr_per_cell_dim"] = tot * 32 / cells
    out["opcode_thread_instr_per_cell_dim"] = {o: round(n * 32 / cells, 3) for o, n in ops.most_common(30)}
    dr = out.get("dram__bytes_read.sum", (0, "byte"))
    dw = out.get("dram__bytes_write.sum", (0, "byte"))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    out["traffic_bytes"] = dr[0] * scale.get(dr[1], 1) + dw[0] * scale.get(dw[1], 1)
    with open(prefix + ".json", "w") as f:
        json.dump(out, f, indent=1)
    with open(prefix + ".txt", "w") as f:
        for k, v in out.items():
            f.write(f"{k}: {v}\n")
    print(json.dumps({k: out[k] for k in ("traffic_bytes", "thread_instr_per_cell_dim")}))


def launches(path, outp):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr = rows[hi]
    ix = {h: i for i, h in enumerate(hdr)}
    tot = collections.Counter()
    cnt = collections.Counter()
    unit = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    for r in rows[hi + 1:]:
        if len(r) < len(hdr) or r[ix["Metric Name"]] != "gpu__time_duration.sum":
            continue
        name = r[ix["Kernel Name"]].split("(")[0][:70]
        tot[name] += float(r[ix["Metric Value"]].replace(",", "")) * unit.get(r[ix["Metric Unit"]], 1e-6)
        cnt[name] += 1
    T = sum(tot.values())
    with open(outp, "w") as f:
        f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none launch list: {path}\n")
        f.write("# cold-cache, serialised per-launch times: compare SHARES, not absolutes\n")
        for k, v in tot.most_common():
            f.write(f"{k:70s} launches={cnt[k]:4d} total_ms={v:12.3f} share={v / T * 100:6.2f}%\n")
    print(open(outp).read())


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], sys.argv[3], sys.argv[4])
    else:
        launches(sys.argv[2], sys.argv[3])
