"""Summarise the per-config ncu captures of tools/ncu_configs.sh into profiles/.

    python tools/ncu_config_summary.py <tag, e.g. r02>

Inputs: gpurun_out/ncu_cfg<N>.csv (ncu --metrics ... --csv of one whole integrator call, every
kernel in the profiler range) and gpurun_out/ncu_cfg<N>.log (tools/ncu_cfg.py's JSON line: the
call's work counters).  Writes profiles/<tag>_ncu_configs.md (one table, every config) and
profiles/ncu_traffic_cfg<N>.json (DRAM bytes of one integrator call, bench.py's
roofline.traffic).  Durations are ncu's (kernels serialised, replayed): shares and counters are
the evidence, the bench's event timing is the performance number.
"""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
SCALE = {"ns": 1e-9, "nsecond": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3,
         "s": 1.0, "second": 1.0}
BYTES = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
F_EVAL, F_NODE, F_SEG = 210, 100, 60


def load(n):
    rows = list(csv.reader(open(os.path.join(OUT, f"ncu_cfg{n}.csv"))))
    hi = next(i for i, r in enumerate(rows) if "Metric Name" in r)
    hdr = rows[hi]
    ix = {h: j for j, h in enumerate(hdr)}
    launches = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) < len(hdr):
            continue
        key = (r[ix["ID"]], r[ix["Kernel Name"]].split("(")[0].replace("void ", "")
               .replace("<unnamed>::", ""))
        unit, val = r[ix["Metric Unit"]], r[ix["Metric Value"]].replace(",", "")
        try:
            v = float(val)
        except ValueError:
            v = None
        if v is not None and unit in SCALE:
            v *= SCALE[unit]
        if v is not None and unit in BYTES:
            v *= BYTES[unit]
        launches.setdefault(key, {})[r[ix["Metric Name"]]] = v
    info = json.loads(open(os.path.join(OUT, f"ncu_cfg{n}.log")).read().strip().splitlines()[-1])
    return launches, info


def load_dram(n):
    rows = list(csv.reader(open(os.path.join(OUT, f"ncu_cfg{n}_dram.csv"))))
    hi = next(i for i, r in enumerate(rows) if "Metric Name" in r)
    hdr = rows[hi]
    ix = {h: j for j, h in enumerate(hdr)}
    launches = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) < len(hdr):
            continue
        key = (r[ix["ID"]], r[ix["Kernel Name"]].split("(")[0].replace("void ", "")
               .replace("<unnamed>::", ""))
        unit, val = r[ix["Metric Unit"]], r[ix["Metric Value"]].replace(",", "")
        v = float(val) * BYTES.get(unit, 1) * SCALE.get(unit, 1)
        launches.setdefault(key, {})[r[ix["Metric Name"]]] = v
    return launches, None


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r02"
    peak = 36.27  # TF/s, measured DFMA peak (profiles/r01_fp64_dmma_mix.json)
    lines = [f"# {tag}: ncu of one whole integrator call per BASELINE config (tools/ncu_configs.sh)",
             "",
             "`python tools/ncu_cfg.py <cfg> <warm> 1 subregion` under `ncu --metrics ...`: after the "
             "warm-up steps, one `rp_compute_potentials` on the full mesh; every kernel of the call "
             "is in the profiler range. Integrator = `k_integrate` item launch + unit launch. "
             "Algorithmic TF/s = the census (evals - skipped) x 210 + r' nodes x 100 + segments x 60 "
             f"over the ncu durations of the two integrator launches; peak {peak} TF/s (DFMA, "
             "measured). ncu durations are serialised replays (`--clock-control none`). DRAM GB/call: "
             "read + write of the integrator launches of one whole-mesh call; ring GB: the whole "
             "history ring (the levels with support are read once with the subregion-major order; the "
             "rest of the traffic is the dense (point, subregion) item arrays). Config 5: the counters "
             "of rank 0's shard of an 8-way split (`tools/ncu_cfg5.sh`; a full call is ~55 s per ncu "
             "replay pass) and the DRAM bytes of its whole call.",
             "",
             "| config | integrator ms (ncu) | share of call | alg. TF/s | frac | FP64 pipe % | "
             "executed FP64 TF/s | DRAM GB/call | ring GB | L2 hit % | L1 hit % | branch uniform % | "
             "sectors/req | threads/instr | warps active % | issue % | regs |",
             "|" + "---|" * 17]
    for n in range(1, 6):
        try:
            launches, info = load(n)
        except Exception as e:  # pragma: no cover
            lines.append(f"| cfg{n} | missing ({e}) |")
            continue
        integ = [m for (i, name), m in launches.items() if name.startswith("k_integrate")]
        tot_t = sum(m.get("gpu__time_duration.sum") or 0 for m in launches.values())
        t = sum(m.get("gpu__time_duration.sum") or 0 for m in integ)
        w = lambda k: sum((m.get(k) or 0) * (m.get("gpu__time_duration.sum") or 0) for m in integ) / t
        s = lambda k: sum(m.get(k) or 0 for m in integ)
        inf = info["info"]
        alg = (inf["evals"] - inf["skipped"]) * F_EVAL + inf["nodes"] * F_NODE + inf["segments"] * F_SEG
        exe = 2 * s("smsp__sass_thread_inst_executed_op_dfma_pred_on.sum") + \
            s("smsp__sass_thread_inst_executed_op_dmul_pred_on.sum") + \
            s("smsp__sass_thread_inst_executed_op_dadd_pred_on.sum")
        dram = s("dram__bytes_read.sum") + s("dram__bytes_write.sum")
        cfg = info["config"]
        if info.get("world", 1) > 1:
            # counters of a shard (rank 0 of info["world"]); DRAM of the whole call separately
            cfg = f"{cfg} (rank 0 of {info['world']})"
            try:
                full, _ = load_dram(n)
                dram = sum((m.get("dram__bytes_read.sum") or 0) + (m.get("dram__bytes_write.sum") or 0)
                           for (i, name), m in full.items() if name.startswith("k_integrate"))
            except Exception:
                dram = float("nan")
        nx = int(cfg.split("-")[1].split("x")[0])
        kap = inf["kappa"]
        alg_dram = (kap + 2) * (nx + 6) ** 2 * 32
        sec = s("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum")
        req = s("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")
        lines.append(
            f"| {cfg} | {1e3 * t:.1f} | {t / tot_t:.3f} | {alg / t / 1e12:.2f} | {alg / t / 1e12 / peak:.3f} | "
            f"{w('sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | {exe / t / 1e12:.2f} | "
            f"{dram / 1e9:.3f} | {alg_dram / 1e9:.3f} | {w('lts__t_sector_hit_rate.pct'):.1f} | "
            f"{w('l1tex__t_sector_hit_rate.pct'):.1f} | "
            f"{w('smsp__sass_average_branch_targets_threads_uniform.pct'):.1f} | {sec / max(req, 1):.2f} | "
            f"{w('smsp__thread_inst_executed_per_inst_executed.ratio'):.2f} | "
            f"{w('sm__warps_active.avg.pct_of_peak_sustained_active'):.1f} | "
            f"{w('smsp__issue_active.avg.pct_of_peak_sustained_active'):.1f} | "
            f"{max(m.get('launch__registers_per_thread') or 0 for m in integ):.0f} |")
        json.dump({"dram_bytes_per_call": dram, "integrator_launches": len(integ),
                   "algorithmic_dram_bytes": alg_dram, "config": cfg,
                   "source": f"profiles/{tag}_ncu_configs.md (tools/ncu_configs.sh, {tag})"},
                  open(os.path.join(PROF, f"ncu_traffic_cfg{n}.json"), "w"), indent=1)
    lines += ["", "Per-launch detail (ncu durations, ms):", ""]
    for n in range(1, 6):
        try:
            launches, _ = load(n)
        except Exception:
            continue
        agg = collections.defaultdict(float)
        for (i, name), m in launches.items():
            agg[name[:60]] += 1e3 * (m.get("gpu__time_duration.sum") or 0)
        lines.append(f"- cfg{n}: " + ", ".join(f"`{k}` {v:.2f}" for k, v in
                                               sorted(agg.items(), key=lambda x: -x[1])[:6]))
    open(os.path.join(PROF, f"{tag}_ncu_configs.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
