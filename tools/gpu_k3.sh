# K3 (pg_compare) on C5 transpose: bench line + the compare launches' time / DRAM bytes / issue
O=gpurun_out/r2/k3; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python bench.py --workload c5t --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_c5t.json 2> $O/bench_c5t.err
python -c "import json;d=json.loads(open('$O/bench_c5t.json').read().strip().splitlines()[-1]);print('%.4g'%d['value'],d['ms_per_step'],d['roofline']['k2_busy_ms_per_step'])"
export PGVC_GRAPH=0 PGVC_COND=host
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active \
    --clock-control none --profile-from-start off -k regex:"pg_compare|pg_gen_inputs|pg_xb" --csv --log-file $O/k3.csv python bench.py --profile --workload c5t > $O/k3.log 2>&1
python - <<'PY'
import csv,collections
rows=list(csv.reader(open('gpurun_out/r2/k3/k3.csv')))
hdr=None;L=collections.defaultdict(dict)
for r in rows:
    if r and r[0]=='ID': hdr=r; continue
    if hdr and len(r)==len(hdr):
        d=dict(zip(hdr,r)); i=int(d['ID']); L[i][d['Metric Name']]=float(d['Metric Value'].replace(',',''));L[i]['name']=d['Kernel Name'][:40]
for i,v in sorted(L.items()):
    t=v['gpu__time_duration.sum']; b=v.get('dram__bytes_read.sum',0)+v.get('dram__bytes_write.sum',0)
    if t>100000: print(v['name'],'%.2f ms'%(t/1e6),'%.0f GB/s'%(b/t),'issue %.0f warps %.0f'%(v['smsp__issue_active.avg.pct_of_peak_sustained_active'],v['sm__warps_active.avg.pct_of_peak_sustained_active']))
PY
