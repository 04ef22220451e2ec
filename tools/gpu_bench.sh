# one GPU session: build, the C2 bench on per-pair streams (default) and on one stream, then
# the ncu launch list + K2 metrics + top-launch capture of one step (tools/profile_round.sh)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python bench.py --steps 20 --warmup 5 --diag > gpurun_out/bench_s0.json 2> gpurun_out/bench_s0.err
tail -4 gpurun_out/bench_s0.err; cat gpurun_out/bench_s0.json
timeout 600 python bench.py --steps 20 --warmup 5 --diag --streams 1 --no-cpu-baseline > gpurun_out/bench_s1.json 2> gpurun_out/bench_s1.err
tail -4 gpurun_out/bench_s1.err; cat gpurun_out/bench_s1.json
if [ "${PROFILE:-1}" = "1" ]; then timeout 1500 bash tools/profile_round.sh gpurun_out/prof c2; fi
