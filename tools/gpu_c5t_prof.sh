# C5 transpose diagnostics: timeline of one check, ncu launch list + K2 metrics
O=gpurun_out/r2/c5t; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 300 python tools/timeline.py c5t 1250 2 > $O/timeline.txt 2>&1; tail -n 3 $O/timeline.txt
export PGVC_GRAPH=0 PGVC_COND=host
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
    --clock-control none --profile-from-start off --csv --log-file $O/launches.csv python bench.py --profile --workload c5t > $O/launches.log 2>&1
tail -n 3 $O/launches.log
