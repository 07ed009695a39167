#!/bin/bash
# Per-CTA phase timestamps of k_apply_walk and k_predict (run under gpurun):
#   tools/clock_run.sh <tag>
set -u
TAG=${1:-clk}
mkdir -p /tmp/clk; DUM_BUILD_CLOCK=/tmp/clk/build DUM_PRED_CLOCK=/tmp/clk/pred timeout 600 \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline > gpurun_out/${TAG}_clk_bench.log 2>&1
python tools/pred_clock.py /tmp/clk/pred > gpurun_out/${TAG}_pred.txt 2>&1
python tools/build_clock.py /tmp/clk/build > gpurun_out/${TAG}_build.txt 2>&1
rm -rf /tmp/clk
ls gpurun_out/ > /dev/null
