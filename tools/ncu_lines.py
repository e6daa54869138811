"""Attribute ncu warp-stall samples of one kernel to CUDA source lines.

usage: python tools/ncu_lines.py <report.ncu-rep> <cubin> <kernel-substring> [top]
Joins `ncu --page source --csv` (SASS, per-address samples) with `nvdisasm -g` line info.
"""
import collections
import csv
import io
import re
import subprocess
import sys

rep, cubin, kname = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = rows[1]
ix = {h: j for j, h in enumerate(hdr)}
samples = {}
execd = {}
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    try:
        a = int(r[ix["Address"]], 16)
    except ValueError:
        continue
    samples[a] = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    execd[a] = int(r[ix["Instructions Executed"]] or 0)
base = min(samples) if samples else 0
samples = {a - base: v for a, v in samples.items()}
execd = {a - base: v for a, v in execd.items()}
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
line = None
infn = False
by_line = collections.Counter()
ex_line = collections.Counter()
n_line = collections.Counter()
for l in dis.splitlines():
    if l.startswith("\t.text.") or l.startswith(".text."):
        infn = kname in l
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        line = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m and infn and line:
        a = int(m.group(1), 16)
        by_line[line] += samples.get(a, 0)
        ex_line[line] += execd.get(a, 0)
        n_line[line] += 1
tot = sum(by_line.values()) or 1
tex = sum(ex_line.values()) or 1
print(f"total samples {tot}, instructions mapped {sum(n_line.values())}")
for (f, ln), s in by_line.most_common(top):
    print(f"{100*s/tot:5.1f}% stall  {100*ex_line[(f, ln)]/tex:5.1f}% exec  {n_line[(f, ln)]:4d} sass  {f}:{ln}")
