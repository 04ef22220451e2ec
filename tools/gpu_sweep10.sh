O=gpurun_out/r2/sweep10; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { tag=$1; wl=$2; shift 2; env "$@" timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]);r=d['roofline'];print('%.4g'%d['value'],d['ms_per_step'],r['k2_busy_ms_per_step'],'frac %.3f'%r['frac'])" || tail -n 3 $O/$tag.err; }
run base c2n PGVC_X=0
run fs16 c2n PGVC_FAST_STEPS=16
run fs4 c2n PGVC_FAST_STEPS=4
run fs32 c2n PGVC_FAST_STEPS=32
run base2 c2n PGVC_X=0
run c1fs16 c1 PGVC_FAST_STEPS=16
run c1 c1 PGVC_X=0
