# one GPU session: build, every gpu test, then the C2 bench in both designs (pairs, N-kernel)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout ${PYT_TIMEOUT:-2400} python -m pytest tests -m gpu -q -x ${PYT_ARGS:-} 2>&1 | tail -40 > gpurun_out/gputest.log
tail -40 gpurun_out/gputest.log
timeout 900 python bench.py --workload c2 --steps 20 --warmup 5 --diag --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
tail -3 gpurun_out/bench_c2.err; cat gpurun_out/bench_c2.json
timeout 900 python bench.py --steps 20 --warmup 5 --diag --workload c2n > gpurun_out/bench_c2n.json 2> gpurun_out/bench_c2n.err
tail -3 gpurun_out/bench_c2n.err; cat gpurun_out/bench_c2n.json
