# one GPU session: VC-literal + divergence tests, then the c2n ncu profile (PGVC_COND=0)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_vcliteral.py tests/test_gpu_dataflow.py -m gpu -q -x 2>&1 | tail -30 > gpurun_out/gputest.log
tail -30 gpurun_out/gputest.log
timeout 1500 bash tools/profile_round.sh gpurun_out/prof_c2n c2n
