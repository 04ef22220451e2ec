# exact-pass block steps per item (PGVC_RERUN_STEPS) on c2n and c2
O=gpurun_out/r2/sweep; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for wl in c2n c2; do for s in 8 4 2 1; do
  PGVC_RERUN_STEPS=$s timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/${wl}_s$s.json 2> $O/${wl}_s$s.err
  echo "$wl steps=$s"; python -c "import json;d=json.load(open('$O/${wl}_s$s.json'));print('%.3g'%d['value'],d['ms_per_step'],d['roofline']['k2_busy_ms_per_step'])"
done; done
