# bench each prebuilt librp variant in variants/ (quick, no profiler)
for v in variants/*.so variants/*.so; do
  cp $v paper_conf_icpp_arumugamrztgi17_b200/librp.so
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/var.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/var.json')); print('$v', round(d['ms_per_step'],2), 'ms/step', round(d['roofline']['frac'],4))"
done
