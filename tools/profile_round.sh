#!/bin/bash
# Profiling recipe (B200_PROFILING.md) for bench.py; run under gpurun.
#   tools/profile_round.sh <tag>
# Writes gpurun_out/<tag>_launches.csv (every launch, device time, cold-cache and
# serialised: compare SHARES) and gpurun_out/<tag>_<kernel>.ncu-rep (--set full).
set -u
TAG=${1:-r01}
KERNELS=${KERNELS:-"k_predict k_apply_walk k_ingest k_chain"}
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_launches.csv $B > gpurun_out/${TAG}_launches.log 2>&1
for k in $KERNELS; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 \
      -o gpurun_out/${TAG}_$k -f $B > gpurun_out/${TAG}_$k.log 2>&1
done
