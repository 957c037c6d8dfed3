"""Stall samples and executed instructions of an ncu --set full report aggregated by CUDA source
line (SASS addresses mapped to lines with nvdisasm -g of the matching cubin).
  python scripts/ncu_lines.py <report.ncu-rep> <object-or-cubin> <kernel-substring> [top]"""
import collections
import csv
import os
import re
import subprocess
import sys
import tempfile

rep, obj, kname = sys.argv[1], sys.argv[2], sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=tmp, capture_output=True)
cubins = [os.path.join(tmp, f) for f in os.listdir(tmp) if f.endswith(".cubin")] or [obj]
addr_line = {}
for cb in cubins:
    txt = subprocess.run(["nvdisasm", "-g", "-c", cb], capture_output=True, text=True).stdout
    cur_fn, cur_line, in_k = None, None, False
    for ln in txt.splitlines():
        m = re.match(r"\s*\.text\.(\S+):", ln)
        if m:
            in_k = kname in m.group(1)
            continue
        if not in_k:
            continue
        m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
        if m:
            cur_line = f"{os.path.basename(m.group(1))}:{m.group(2)}"
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
        if m and cur_line:
            addr_line[int(m.group(1), 16)] = cur_line
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out))
hdr = rows[1]
base = None  # ncu lists absolute addresses: rebase to the kernel's first instruction
ix = {h: i for i, h in enumerate(hdr)}
stall_cols = [h for h in hdr if h.startswith("stall_")]
agg = collections.defaultdict(lambda: collections.Counter())
tot = collections.Counter()
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    try:
        a = int(r[ix["Address"]], 16)
    except ValueError:
        continue
    if base is None:
        base = a
    a -= base
    line = addr_line.get(a, "?")
    c = agg[line]
    c["samples"] += int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    c["inst"] += int(r[ix["Instructions Executed"]] or 0)
    for h in stall_cols:
        v = float(r[ix[h]] or 0)
        c[h] += v
        tot[h] += v
    tot["samples"] += int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    tot["inst"] += int(r[ix["Instructions Executed"]] or 0)
print(f"mapped {len(addr_line)} addresses; total samples {tot['samples']}, warp instructions {tot['inst']}")
print("top stall reasons:", {h: round(v / max(1, tot['samples']), 3) for h, v in tot.most_common() if h.startswith('stall_')} )
for line, c in sorted(agg.items(), key=lambda kv: -kv[1]["samples"])[:top]:
    reasons = sorted(((c[h], h[6:]) for h in stall_cols if c[h] > 0), reverse=True)[:4]
    print(f"{line:28s} samples {100.0 * c['samples'] / max(1, tot['samples']):5.1f}%  inst {100.0 * c['inst'] / max(1, tot['inst']):5.1f}%  "
          + " ".join(f"{n}={100.0 * v / max(1, c['samples']):.0f}%" for v, n in reasons))
