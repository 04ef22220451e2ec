#!/bin/bash
# Run on the GPU box: `--set full` captures of chosen evaluation-kernel launches of one
# bench step (indices count pgk_eval launches only, as in k2_metrics.csv).
#   tools/capture_k2.sh OUT WORKLOAD IDX [IDX ...]
set -u
export PGVC_GRAPH=0 PGVC_COND=host   # (the launches the conditional nodes run, as plain launches ncu can profile)
OUT=$1; WL=$2; shift 2
mkdir -p "$OUT/src"
for IDX in "$@"; do
  PGVC_DUMP_SRC="$PWD/$OUT/src" timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
      -k regex:pgk_eval -s "$IDX" -c 1 -o "$OUT/k2_$IDX" python bench.py --profile --workload "$WL" > "$OUT/k2_$IDX.log" 2>&1
done
echo done
