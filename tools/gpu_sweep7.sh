O=gpurun_out/r2/sweep7; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { tag=$1; wl=$2; shift 2; env "$@" timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]);r=d['roofline'];print('%.4g'%d['value'],d['ms_per_step'],r['k2_busy_ms_per_step'],'frac %.3f'%r['frac'])" || tail -n 3 $O/$tag.err; }
run c2n c2n PGVC_X=0
run c2n_rc c2n PGVC_RC_INLINE=1
run c2 c2 PGVC_X=0
run c2_rc c2 PGVC_RC_INLINE=1
run c3 c3 PGVC_X=0
run c3_rc c3 PGVC_RC_INLINE=1
run c2n_b c2n PGVC_X=0
