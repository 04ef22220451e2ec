# build, all gpu tests (stop at first failure), then bench lines for the given workloads
O=${OUT:-gpurun_out/r2/cb}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout ${PYT_TIMEOUT:-1800} python -m pytest tests -m gpu -q -x ${PYT_ARGS:-} 2>&1 | tail -30 > $O/gputest.log; tail -n 8 $O/gputest.log
for wl in ${WLS:-c2n}; do
  timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/bench_$wl.json 2> $O/bench_$wl.err
  echo "$wl"; python -c "import json;d=json.loads(open('$O/bench_$wl.json').read().strip().splitlines()[-1]);print('%.4g'%d['value'],d['ms_per_step'],d['roofline']['k2_busy_ms_per_step'])" || tail -n 5 $O/bench_$wl.err
done
