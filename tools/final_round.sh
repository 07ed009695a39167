#!/bin/bash
# Round-end measurement (run under gpurun): GPU tests, smoke(), the default
# bench line (+ --verify), the reference arm, the ncu launch list and
# --set full captures.
#   tools/final_round.sh <tag>
set -u
TAG=${1:-final}
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_tests.log 2>&1
echo "tests_rc=$?" >> gpurun_out/${TAG}_tests.log
cp gpurun_out/path_counters.json gpurun_out/${TAG}_paths.json 2>/dev/null
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/${TAG}_smoke.log 2>&1
timeout 600 python -m pytest tests/test_um_runtime.py tests/test_alloc_hook.py -m gpu -q -s > gpurun_out/${TAG}_um.log 2>&1
timeout 600 python bench.py --fast-windows --no-migration --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_fast.log 2>&1
timeout 600 python bench.py --graph --no-migration --no-cpu-baseline > gpurun_out/${TAG}_bench_graph.log 2>&1
timeout 900 python bench.py --verify > gpurun_out/${TAG}_bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_ref.log 2>&1
nproc > gpurun_out/${TAG}_nproc.txt; lscpu | head -20 >> gpurun_out/${TAG}_nproc.txt
bash tools/profile_round.sh ${TAG}
