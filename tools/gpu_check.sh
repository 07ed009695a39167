#!/bin/bash
# Iteration check (run under gpurun): the -m gpu suite, then the default bench line.
#   tools/gpu_check.sh <tag> [pytest -k expr]
set -u
T=${1:-chk}
K=${2:-}
if [ -n "$K" ]; then
  timeout -k 10 1500 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/${T}_tests.log 2>&1
else
  timeout -k 10 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_tests.log 2>&1
fi
echo "rc=$?" >> gpurun_out/${T}_tests.log
timeout -k 10 600 python bench.py --no-migration --no-cpu-baseline > gpurun_out/${T}_bench.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_bench.log
