# one GPU session: build, selected gpu tests ($TESTS), timeline of c2n, bench c2n (and $WLS)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
if [ -n "${TESTS:-}" ]; then
  timeout ${PYT_TIMEOUT:-1200} python -m pytest $TESTS -m gpu -q -x 2>&1 | tail -30 > gpurun_out/gputest_q.log
  tail -30 gpurun_out/gputest_q.log
fi
timeout 300 python tools/timeline.py c2n 64 3 > gpurun_out/tl_c2n.txt 2>&1
for wl in ${WLS:-c2n}; do
  timeout 900 python bench.py --steps 20 --warmup 5 --diag --workload $wl --no-cpu-baseline > gpurun_out/bq_$wl.json 2> gpurun_out/bq_$wl.err
  tail -3 gpurun_out/bq_$wl.err; head -c 700 gpurun_out/bq_$wl.json; echo
done
