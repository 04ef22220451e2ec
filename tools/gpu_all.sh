# one GPU session: build, every gpu test, then the C2 bench (no profile)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout ${PYT_TIMEOUT:-2400} python -m pytest tests -m gpu -q ${PYT_ARGS:-} 2>&1 | tail -60 > gpurun_out/gputest.log
tail -60 gpurun_out/gputest.log
timeout 900 python bench.py --steps 20 --warmup 5 --diag > gpurun_out/bench_s0.json 2> gpurun_out/bench_s0.err
tail -4 gpurun_out/bench_s0.err; cat gpurun_out/bench_s0.json
