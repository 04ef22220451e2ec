# exact-pass block steps per item for blocks of >= 512 threads (PGVC_RERUN_STEPS_L), and 16 overall
O=gpurun_out/r2/sweep2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { tag=$1; shift; env "$@" timeout 600 python bench.py --workload c2n --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.load(open('$O/$tag.json'));print('%.3g'%d['value'],d['ms_per_step'],d['roofline']['k2_busy_ms_per_step'])"; }
run base PGVC_RERUN_STEPS=8
run L4 PGVC_RERUN_STEPS_L=4
run L2 PGVC_RERUN_STEPS_L=2
run L1 PGVC_RERUN_STEPS_L=1
run s16 PGVC_RERUN_STEPS=16
run s16L4 PGVC_RERUN_STEPS=16 PGVC_RERUN_STEPS_L=4
