# c3 with and without store-time claims; c2n default (fast steps 2); remaining configs' bench lines
O=gpurun_out/r2/sweep4; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { tag=$1; wl=$2; shift 2; env "$@" timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  echo "$tag"; python -c "import json;d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]);r=d['roofline'];print('%.4g'%d['value'],d['ms_per_step'],r['k2_busy_ms_per_step'],'frac %.3f alu %.3f counted %.3f'%(r['frac'],r['frac_of_alu_pipe'],r['frac_counted_ops']))" || tail -n 3 $O/$tag.err; }
run c3cas0 c3 PGVC_CAS=0
run c3 c3 PGVC_X=0
run c2n c2n PGVC_X=0
run c2ncas0 c2n PGVC_CAS=0
run c4 c4 PGVC_X=0
run c5t c5t PGVC_X=0
run c5m c5m PGVC_X=0
