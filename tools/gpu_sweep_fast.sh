# optimistic-pass block steps per item for blocks of >= 256 threads (PGVC_FAST_STEPS_L); c3 noise
O=gpurun_out/r2/sweep3; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { tag=$1; wl=$2; shift 2; env "$@" timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]);print('%.4g'%d['value'],d['ms_per_step'],d['roofline']['k2_busy_ms_per_step'])"; }
run base c2n PGVC_X=0
run f2 c2n PGVC_FAST_STEPS_L=2
run f4 c2n PGVC_FAST_STEPS_L=4
run f8 c2n PGVC_FAST_STEPS_L=8
run base2 c2n PGVC_X=0
run c3a c3 PGVC_X=0
run c3b c3 PGVC_X=0
