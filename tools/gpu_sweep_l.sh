# exact-pass steps for blocks of >= 256 threads (PGVC_RERUN_L_MIN / PGVC_RERUN_STEPS_L)
O=gpurun_out/r2/sweep5; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { tag=$1; wl=$2; shift 2; env "$@" timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]);r=d['roofline'];print('%.4g'%d['value'],d['ms_per_step'],r['k2_busy_ms_per_step'],'frac %.3f'%r['frac'])" || tail -n 3 $O/$tag.err; }
run base c2n PGVC_X=0
run m256l4 c2n PGVC_RERUN_L_MIN=256
run m256l2 c2n PGVC_RERUN_L_MIN=256 PGVC_RERUN_STEPS_L=2
run m128l4 c2n PGVC_RERUN_L_MIN=128
run base2 c2n PGVC_X=0
run seedh0 c2n PGVC_SEEDH=0
run c3 c3 PGVC_X=0
run c3seedh0 c3 PGVC_SEEDH=0
run c3b c3 PGVC_X=0
