# one GPU session: build, INT32 peak, pytest -m gpu, C2 bench on one stream and on per-pair streams
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
python -c "
import torch
from paper_conf_ipps_lig12_b200 import pgvc
torch.cuda.init()
print('INT32', pgvc.measure_int32_peak())
" 2>&1 | tail -3
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -30 > gpurun_out/gputest.log
tail -5 gpurun_out/gputest.log
PGVC_TRACE=1 timeout 600 python bench.py --steps 20 --warmup 5 --diag --no-cpu-baseline > gpurun_out/bench1.json 2> gpurun_out/bench1.err
tail -3 gpurun_out/bench1.err; cat gpurun_out/bench1.json
timeout 600 python bench.py --steps 20 --warmup 5 --diag --no-cpu-baseline --streams 0 > gpurun_out/bench0.json 2> gpurun_out/bench0.err
tail -3 gpurun_out/bench0.err; cat gpurun_out/bench0.json
