# one GPU session: build, edges/parity/bank tests, then the C1 / C3 / C2 benches
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 1500 python -m pytest tests/test_gpu_edges.py tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -8 > gpurun_out/gputest.log
tail -8 gpurun_out/gputest.log
for w in c1 c3 c2n; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bw_$w.json 2> gpurun_out/bw_$w.err; python -c "import json; d=json.load(open('gpurun_out/bw_$w.json')); print('$w', '%.3e' % d['value'], '%.3f ms' % d['ms_per_step'], 'k2 %.3f' % d['roofline']['k2_busy_ms_per_step'])"; done
