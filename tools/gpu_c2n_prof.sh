# c2n: bench line, one check's per-launch timeline, ncu launch list + K2 metrics + top capture
# (host-decided conditional blocks: the production launch set); then c3 bench + timeline
O=gpurun_out/r2/c2n; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python bench.py --workload c2n --steps 20 --warmup 5 --diag > $O/bench.json 2> $O/bench.err; tail -n 2 $O/bench.err; cat $O/bench.json
timeout 300 python tools/timeline.py c2n 64 3 > $O/timeline.txt 2>&1; tail -n 5 $O/timeline.txt
[ -n "${NOPROF:-}" ] || timeout 1200 bash tools/profile_round.sh $O/prof c2n
O3=gpurun_out/r2/c3; mkdir -p $O3
timeout 600 python bench.py --workload c3 --steps 10 --warmup 3 --diag > $O3/bench.json 2> $O3/bench.err; tail -n 2 $O3/bench.err; cat $O3/bench.json
timeout 300 python tools/timeline.py c3 64 2 > $O3/timeline.txt 2>&1; tail -n 5 $O3/timeline.txt
