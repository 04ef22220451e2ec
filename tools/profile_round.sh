#!/bin/bash
# Run on the GPU box (gpurun): ncu evidence for one bench step of the headline workload.
#   1. every launch of one step with its device time (cold-cache, serialised: compare shares)
#   2. DRAM bytes and time of every evaluation-kernel launch (roofline "traffic")
#   3. one `--set full` capture of the top evaluation-kernel launch (source-level, -lineinfo)
set -u
# ncu cannot profile the kernel nodes of a graph that has conditional nodes: profile the checks
# eagerly, the host deciding each conditional block from its flag word - the same launches the
# graphs run
export PGVC_GRAPH=0 PGVC_COND=host
OUT=${1:-gpurun_out/prof}
WL=${2:-c2}
mkdir -p "$OUT/src"
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file "$OUT/launches.csv" python bench.py --profile --workload "$WL" > "$OUT/launches.log" 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active \
    --clock-control none --profile-from-start off -k regex:pgk_eval --csv \
    --log-file "$OUT/k2_metrics.csv" python bench.py --profile --workload "$WL" > "$OUT/k2_metrics.log" 2>&1
# the longest evaluation-kernel launch of the metrics pass (same filter => same launch index)
SKIP=${K2_SKIP:-$(python - "$OUT/k2_metrics.csv" <<'PY'
import csv, sys
best, idx, seen = -1.0, 0, {}
for r in csv.reader(open(sys.argv[1])):
    if len(r) > 14 and r[0].isdigit() and r[12] == "gpu__time_duration.sum":
        i = int(r[0])
        if i not in seen:
            seen[i] = len(seen)
        v = float(r[14].replace(",", ""))
        if v > best:
            best, idx = v, seen[i]
print(idx)
PY
)}
echo "k2 top launch index: $SKIP"
PGVC_DUMP_SRC="$PWD/$OUT/src" ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k regex:pgk_eval -s "$SKIP" -c 1 -o "$OUT/k2_top" python bench.py --profile --workload "$WL" > "$OUT/k2_top.log" 2>&1
echo done
