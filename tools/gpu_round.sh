#!/bin/bash
# One GPU iteration (run under gpurun): parity tests, bench, ncu launch list and
# a --set full capture of the kernels in $KERNELS.
#   tools/gpu_round.sh <tag> [pytest -k expr]
set -u
TAG=${1:-r01}
KEXPR=${2:-}
KERNELS=${KERNELS:-"k_predict"}
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
if [ -n "$KEXPR" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -k "$KEXPR" > gpurun_out/${TAG}_tests.log 2>&1
else
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_tests.log 2>&1
fi
echo "tests_rc=$?" >> gpurun_out/${TAG}_tests.log
timeout 600 python bench.py ${BENCH_ARGS:-} > gpurun_out/${TAG}_bench.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_launches.csv $B > gpurun_out/${TAG}_launches.log 2>&1
for k in $KERNELS; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 \
      -o gpurun_out/${TAG}_$k -f $B > gpurun_out/${TAG}_$k.log 2>&1
done
