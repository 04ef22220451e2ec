# one GPU session: VC-literal, data-flow and sequence tests
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 1200 python -m pytest tests/test_gpu_vcliteral.py tests/test_gpu_sequence.py tests/test_gpu_dataflow.py -m gpu -q -x 2>&1 | tail -30 > gpurun_out/gputest.log
tail -30 gpurun_out/gputest.log
