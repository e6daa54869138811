# Same bench command plain and under an ncu launch list (per-launch durations), to compare the
# integrator's per-step time in the two settings (shares must agree; absolutes are checked here).
python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tc_plain.json 2> gpurun_out/tc_plain.err
python -c "
import json; d=json.load(open('gpurun_out/tc_plain.json')); print('plain', d['ms_per_step'], d['kernel_ms_per_step']['integrate_ms'], d['kernel_ms_per_step']['units_ms'], d['clocks'])"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/tc_launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tc_ncu.json 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.DictReader(open('gpurun_out/tc_launches.csv')) if r.get('Metric Name')=='gpu__time_duration.sum']
for r in rows:
    if 'k_integrate' in r['Kernel Name']:
        print(r['ID'], r['Kernel Name'][:30], r['Metric Value'], r['Metric Unit'])
PY
python -c "
import json; d=json.loads(open('gpurun_out/tc_ncu.json').read().strip().splitlines()[-1]); print('under ncu (events)', d['ms_per_step'], d['kernel_ms_per_step']['integrate_ms'], d['kernel_ms_per_step']['units_ms'])"
