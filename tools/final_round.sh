#!/bin/bash
# Round-end measurement (run under gpurun): GPU tests, smoke(), the default
# bench line, the ncu launch list and --set full captures, per-CTA clocks.
#   tools/final_round.sh <tag>
set -u
TAG=${1:-final}
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_tests.log 2>&1
echo "tests_rc=$?" >> gpurun_out/${TAG}_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/${TAG}_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/${TAG}_bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_ref.log 2>&1
nproc > gpurun_out/${TAG}_nproc.txt; lscpu | head -20 >> gpurun_out/${TAG}_nproc.txt
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_launches.csv $B > gpurun_out/${TAG}_launches.log 2>&1
for k in k_predict k_apply k_walk k_chain k_ingest; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 \
      -o gpurun_out/${TAG}_$k -f $B > gpurun_out/${TAG}_$k.log 2>&1
done
bash tools/clock_run.sh ${TAG}
