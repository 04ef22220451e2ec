# one GPU session: the timeline of one c2n / c1 check, then a re-run-steps sweep of c2n
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 300 python tools/timeline.py c2n 64 3 > gpurun_out/tl_c2n.txt 2>&1
timeout 300 python tools/timeline.py c1 64 3 > gpurun_out/tl_c1.txt 2>&1
for s in 2 4 8; do
  PGVC_RERUN_STEPS=$s timeout 600 python bench.py --steps 10 --warmup 3 --workload c2n --no-cpu-baseline > gpurun_out/rs$s.json 2> gpurun_out/rs$s.err
done
grep -h '"value"' gpurun_out/rs*.json | cut -c1-200
