# one GPU session: selected tests, then a knob sweep over workloads ($KNOB in $VALS, $WLS)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
if [ -n "${TESTS:-}" ]; then
  timeout ${PYT_TIMEOUT:-1200} python -m pytest $TESTS -m gpu -q -x 2>&1 | tail -30 > gpurun_out/gputest_q.log
  tail -5 gpurun_out/gputest_q.log
fi
for wl in $WLS; do for v in $VALS; do
  env $KNOB=$v timeout 600 python bench.py --steps 20 --warmup 5 --workload $wl --no-cpu-baseline > gpurun_out/sw_${wl}_$v.json 2> gpurun_out/sw_${wl}_$v.err
  echo "$wl $KNOB=$v $(python -c "import json;d=json.load(open('gpurun_out/sw_${wl}_$v.json'));print('%.3e'%d['value'], d['ms_per_step'], d['roofline']['k2_busy_ms_per_step'])")"
done; done
