# one GPU session: build, then the given pytest selection (default: every gpu test)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout ${PYT_TIMEOUT:-1500} python -m pytest ${@:-tests} -m gpu -x -q 2>&1 | tail -40 > gpurun_out/gputest.log
tail -40 gpurun_out/gputest.log
