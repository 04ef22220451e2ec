# ncu launch list of one bench step of workload $1 (time, DRAM bytes, issue, warps) + a summary
WL=${1:-c3}; O=gpurun_out/r2/ll_$WL; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
export PGVC_GRAPH=0 PGVC_COND=host
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active \
    --clock-control none --profile-from-start off --csv --log-file $O/launches.csv python bench.py --profile --workload $WL > $O/launches.log 2>&1
python - "$O/launches.csv" <<'PY'
import csv,collections,sys
rows=list(csv.reader(open(sys.argv[1])))
hdr=None;L=collections.defaultdict(dict)
for r in rows:
    if r and r[0]=='ID': hdr=r; continue
    if hdr and len(r)==len(hdr):
        d=dict(zip(hdr,r)); i=int(d['ID']); L[i][d['Metric Name']]=float(d['Metric Value'].replace(',',''))
        L[i]['name']=d['Kernel Name'].split('(')[0][:28]; L[i]['grid']=d['Grid Size']; L[i]['block']=d['Block Size']
agg=collections.defaultdict(lambda:[0,0,0.0,0.0])
for v in L.values():
    a=agg[v['name']]; t=v['gpu__time_duration.sum']; a[0]+=1; a[1]+=t; a[2]+=v.get('dram__bytes_read.sum',0)+v.get('dram__bytes_write.sum',0); a[3]+=t*v.get('smsp__issue_active.avg.pct_of_peak_sustained_active',0)
tot=sum(a[1] for a in agg.values())
for k,a in sorted(agg.items(), key=lambda kv:-kv[1][1]):
    print('%-30s n=%4d %8.3f ms %5.1f%% %7.0f GB/s issue %4.1f'%(k,a[0],a[1]/1e6,100*a[1]/tot,a[2]/a[1] if a[1] else 0,a[3]/a[1] if a[1] else 0))
top=sorted(L.items(), key=lambda kv:-kv[1]['gpu__time_duration.sum'])[:12]
for i,v in top: print(i,v['name'],v['grid'],v['block'],'%.3f ms'%(v['gpu__time_duration.sum']/1e6),'issue %.0f warps %.0f'%(v['smsp__issue_active.avg.pct_of_peak_sustained_active'],v['sm__warps_active.avg.pct_of_peak_sustained_active']))
PY
