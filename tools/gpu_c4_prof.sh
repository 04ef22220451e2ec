# C4 diagnostics: timeline of each check, ncu launch list with time / DRAM / issue
O=gpurun_out/r2/c4; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 300 python tools/timeline.py c4 64 2 > $O/timeline.txt 2>&1; grep -v timeline $O/timeline.txt | tail -n 12
export PGVC_GRAPH=0 PGVC_COND=host
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active \
    --clock-control none --profile-from-start off --csv --log-file $O/launches.csv python bench.py --profile --workload c4 > $O/launches.log 2>&1
tail -n 2 $O/launches.log
