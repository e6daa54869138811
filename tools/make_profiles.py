"""Summarise gpurun_out/ ncu outputs into profiles/ (committed evidence).

    python tools/make_profiles.py <round tag, e.g. r01>

Reads gpurun_out/launches.csv (ncu --metrics gpu__time_duration.sum launch list) and
gpurun_out/prof_integrate.ncu-rep (ncu --set full of k_integrate); writes
profiles/<tag>_launches.md, profiles/<tag>_ncu_integrate.md and profiles/ncu_integrate.json
(the per-launch DRAM traffic bench.py reports as roofline.traffic).
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
BYTES = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}

# ---------------------------------------------------------------- launch list
rows = list(csv.reader(open(os.path.join(OUT, "launches.csv"))))
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hi]
ix = {h: j for j, h in enumerate(hdr)}
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[hi + 1:]:
    if len(r) < len(hdr) or r[ix["Metric Name"]] != "gpu__time_duration.sum":
        continue
    name = r[ix["Kernel Name"]].split("(")[0].replace("void ", "").replace("<unnamed>::", "")
    name = name[:70]
    agg[name][0] += 1
    agg[name][1] += float(r[ix["Metric Value"]].replace(",", "")) * SCALE[r[ix["Metric Unit"]]]
tot = sum(v[1] for v in agg.values())
lines = [f"# {tag}: ncu launch list of `bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline`",
         "(gpu__time_duration.sum, --clock-control none; cold-cache and serialised: compare shares, not absolutes)",
         "", "| kernel | launches | total ms | share |", "|---|---|---|---|"]
for k, (n, ms) in sorted(agg.items(), key=lambda x: -x[1][1]):
    lines.append(f"| `{k}` | {n} | {ms:.3f} | {100 * ms / tot:.2f}% |")
open(os.path.join(PROF, f"{tag}_launches.md"), "w").write("\n".join(lines) + "\n")

# ---------------------------------------------------------------- full capture of k_integrate
# one integrator call = the item launch + the subtree-unit launch (UNIT = true); the capture
# holds both launches of one step
rep = os.path.join(OUT, "prof_integrate.ncu-rep")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
launches = [{k: (u, v) for k, u, v in zip(rows[0], rows[1], r)} for r in rows[2:] if len(r) == len(rows[0])]


def num(d, k):
    u, v = d[k]
    return float(v.replace(",", "")) * BYTES.get(u, 1)



keys = [("duration (ms, under ncu)", "gpu__time_duration.sum"),
        ("registers / thread", "launch__registers_per_thread"),
        ("achieved warps / SM (% of 64)", "sm__warps_active.avg.pct_of_peak_sustained_active"),
        ("issue active %", "smsp__issue_active.avg.pct_of_peak_sustained_active"),
        ("FP64 pipe active %", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
        ("threads / warp instruction", "smsp__thread_inst_executed_per_inst_executed.ratio"),
        ("warp instructions", "smsp__inst_executed.sum"),
        ("L1 data-pipe wavefronts % (L1->RF bandwidth)", "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed"),
        ("L1 global-load requests", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum"),
        ("L1 global-load sectors", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"),
        ("L1 hit rate %", "l1tex__t_sector_hit_rate.pct"),
        ("L2 hit rate %", "lts__t_sector_hit_rate.pct"),
        ("DRAM read", "dram__bytes_read.sum"), ("DRAM write", "dram__bytes_write.sum")]
names = [d["Kernel Name"][1].split("(")[0].replace("void ", "").replace("<unnamed>::", "")[:60]
         for d in launches]
lines = [f"# {tag}: ncu --set full of the integrator (cfg2 64x64 bend, one step after warm-up)", "",
         "One integrator call = the item launch (`k_integrate<..., false>`) + the subtree-unit launch",
         "(`k_integrate<..., true>`, deep trees split at level 12).", "",
         "| metric | " + " | ".join(f"`{n}`" for n in names) + " |",
         "|---|" + "---|" * len(launches)]
for label, k in keys:
    if all(k in d for d in launches):
        lines.append(f"| {label} (`{k}`) | " + " | ".join(f"{d[k][1]} {d[k][0]}" for d in launches) + " |")
for i, d in enumerate(launches):
    stalls = []
    for k, (u, v) in d.items():
        if "smsp__average_warps_issue_stalled" in k and k.endswith("_per_issue_active.ratio"):
            try:
                stalls.append((float(v), k.replace("smsp__average_warps_issue_stalled_", "").replace(
                    "_per_issue_active.ratio", "")))
            except ValueError:
                pass
    stalls.sort(reverse=True)
    lines += ["", f"Warp stall reasons of `{names[i]}` (cycles per issued instruction):", ""]
    lines += [f"- {name}: {v:.3f}" for v, name in stalls[:8]]
dram = sum(num(d, "dram__bytes_read.sum") + num(d, "dram__bytes_write.sum") for d in launches)
dur = sum(num(d, "gpu__time_duration.sum") for d in launches)
lines += ["", f"DRAM traffic per integrator call (all {len(launches)} launches, read + write): {dram:.0f} bytes"]
open(os.path.join(PROF, f"{tag}_ncu_integrate.md"), "w").write("\n".join(lines) + "\n")
json.dump({"round": tag, "kernel": "k_integrate (items + units)", "launches": len(launches),
           "dram_bytes_per_launch": dram, "dram_bytes_per_call": dram,
           "duration_ms_under_ncu": dur},
          open(os.path.join(PROF, "ncu_integrate.json"), "w"), indent=1)
print(open(os.path.join(PROF, f"{tag}_launches.md")).read())
print("\n".join(lines))
