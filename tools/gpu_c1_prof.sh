# C1 diagnostics: bench line, per-launch timeline of one check, ncu launch list + K2 metrics
O=gpurun_out/r2/c1; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python bench.py --workload c1 --steps 20 --warmup 5 --diag > $O/bench.json 2> $O/bench.err; tail -n 3 $O/bench.err; cat $O/bench.json
timeout 300 python tools/timeline.py c1 64 3 > $O/timeline.txt 2>&1; tail -n 80 $O/timeline.txt
[ -n "${NOPROF:-}" ] || timeout 1200 bash tools/profile_round.sh $O/prof c1
