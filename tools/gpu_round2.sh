# one GPU session (round 2): build, every gpu test, smoke, bench lines for every config,
# then the ncu evidence of the headline (profile_round.sh)
set -x
O=${OUT:-gpurun_out/r2}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
if [ -z "${SKIP_TESTS:-}" ]; then
timeout ${PYT_TIMEOUT:-2400} python -m pytest tests -m gpu -q ${PYT_ARGS:-} 2>&1 | tail -40 > $O/gputest.log
tail -15 $O/gputest.log
fi
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -2 $O/smoke.log
for wl in ${WLS:-c2n c2 c1 c3 c4 c5t c5m}; do
  timeout 900 python bench.py --workload $wl --steps 20 --warmup 5 --diag > $O/bench_$wl.json 2> $O/bench_$wl.err
  tail -2 $O/bench_$wl.err; cat $O/bench_$wl.json
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; cat $O/bench_ref.json
[ -n "${NOPROF:-}" ] || timeout 1500 bash tools/profile_round.sh $O/prof c2n
ls $O $O/prof
