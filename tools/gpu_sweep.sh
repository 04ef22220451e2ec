# one GPU session: tuning sweep of the c2n bench (env knobs), value per setting
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "PGVC_RERUN_STEPS=8" "PGVC_RERUN_STEPS=1" "PGVC_RERUN_STEPS=2" "PGVC_RERUN_STEPS=4" "PGVC_MS=4" "PGVC_MS=16" "PGVC_VT2_MIN=0" "PGVC_TARGET_REGS=48"; do
  env $cfg timeout 600 python bench.py --workload ${WL:-c2n} --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/sweep.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/sweep.json')); print('$cfg', '%.4e' % d['value'], '%.3f ms' % d['ms_per_step'], 'k2 %.3f' % d['roofline']['k2_busy_ms_per_step'])"
done
