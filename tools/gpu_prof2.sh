# one GPU session: ncu evidence (launch list, K2 metrics, top K2 launch) for c1 and c2n
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for wl in ${WLS:-c1 c2n}; do
  timeout 1500 bash tools/profile_round.sh gpurun_out/prof_$wl $wl
done
