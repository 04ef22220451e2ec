O=gpurun_out/r2/sweep9; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_round2.py tests/test_gpu_benchconfig.py -q -m gpu -x 2>&1 | tail -3
run() { tag=$1; wl=$2; shift 2; env "$@" timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]);r=d['roofline'];print('%.4g'%d['value'],d['ms_per_step'],r['k2_busy_ms_per_step'],'frac %.3f'%r['frac'])" || tail -n 3 $O/$tag.err; }
run new c2n PGVC_X=0
run old c2n PGVC_PACK_OLD=1
run new2 c2n PGVC_X=0
run old2 c2n PGVC_PACK_OLD=1
run c1new c1 PGVC_X=0
run c1old c1 PGVC_PACK_OLD=1
