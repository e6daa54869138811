"""Per-CUDA-source-line warp-stall samples and executed instructions of a profiled kernel,
from the report itself (`ncu --page source --print-source cuda,sass`).

usage: python tools/ncu_lines.py <report.ncu-rep> [top] [--ranges a-b:name,c-d:name]
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 40
ranges = []
for a in sys.argv:
    if a.startswith("--ranges="):
        for r in a.split("=", 1)[1].split(","):
            span, name = r.split(":")
            lo, hi = span.split("-")
            ranges.append((int(lo), int(hi), name))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--print-source", "cuda,sass", "--csv"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None
res = []
fname = None
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and r and r[0].isdigit():
        try:
            stall, ex, thr = int(r[4] or 0), int(r[7] or 0), int(r[8] or 0)
        except ValueError:  # source text with unescaped quotes: take the numbers from the end
            try:
                k = len(r) - len(hdr)
                stall, ex, thr = int(r[4 + k] or 0), int(r[7 + k] or 0), int(r[8 + k] or 0)
            except (ValueError, IndexError):
                continue
        res.append((fname, int(r[0]), r[1][:70], stall, ex, thr))
tot_s = sum(x[3] for x in res) or 1
tot_e = sum(x[4] for x in res) or 1
tot_t = sum(x[5] for x in res) or 1
print(f"samples {tot_s}  warp-instr {tot_e}  thread-instr {tot_t}  avg threads {tot_t / tot_e:.1f}")
for f, ln, src, s, e, t in sorted(res, key=lambda x: -x[3])[:top]:
    print(f"{100*s/tot_s:5.1f}% stall {100*e/tot_e:5.1f}% exec thr {t/max(e,1):4.1f}  {f}:{ln}  {src}")
if ranges:
    print("--- ranges (potentials.cu lines)")
    for lo, hi, name in ranges:
        s = sum(x[3] for x in res if x[0] == "potentials.cu" and lo <= x[1] <= hi)
        e = sum(x[4] for x in res if x[0] == "potentials.cu" and lo <= x[1] <= hi)
        t = sum(x[5] for x in res if x[0] == "potentials.cu" and lo <= x[1] <= hi)
        print(f"{name:>12}: {100*s/tot_s:5.1f}% stall {100*e/tot_e:5.1f}% exec  thr {t/max(e,1):4.1f}")
