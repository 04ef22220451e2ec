# one GPU session: locate the PGVC_SPREAD=2 crash, then c2n with PGVC_SPREAD 0/1 alternating
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
PGVC_SPREAD=2 PGVC_TRACE=1 timeout 120 python -X faulthandler tools/timeline.py c1 8 2 > gpurun_out/dbg_spread2.txt 2>&1
echo "rc=$?"; tail -30 gpurun_out/dbg_spread2.txt
PGVC_SPREAD=2 PGVC_GRAPH=0 timeout 120 python -X faulthandler tools/timeline.py c1 8 2 > gpurun_out/dbg_spread2b.txt 2>&1
echo "rc=$?"; tail -5 gpurun_out/dbg_spread2b.txt
for r in 1 2; do for v in 0 1; do
  PGVC_SPREAD=$v timeout 600 python bench.py --steps 20 --warmup 5 --workload c2n --no-cpu-baseline > gpurun_out/sa_$v.json 2>/dev/null
  echo "c2n SPREAD=$v $(python -c "import json;d=json.load(open('gpurun_out/sa_$v.json'));print('%.3e'%d['value'], d['ms_per_step'])")"
done; done
