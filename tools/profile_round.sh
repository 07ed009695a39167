#!/bin/bash
# Profiling recipe (B200_PROFILING.md) for bench.py; run under gpurun.
#   tools/profile_round.sh <tag> [kernel ...]
# Writes gpurun_out/<tag>_launches.csv (every launch: device time + DRAM bytes;
# cold-cache and serialised: compare SHARES, not absolutes) and, per kernel,
# gpurun_out/<tag>_<kernel>.ncu-rep (--set full, one launch after warm-up).
# Kernels are matched on the demangled name ("dum::k_walk<" does not match
# k_walk_slow).
set -u
TAG=${1:-r02}
shift
KERNELS=${*:-"k_predict k_build_exec k_chain k_ingest k_build_prep"}
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_launches.csv $B > gpurun_out/${TAG}_launches.log 2>&1
for k in $KERNELS; do
  case $k in
    k_walk|k_apply|k_build_exec|k_predict) pat="dum::$k<" ;;
    *) pat="dum::$k(" ;;
  esac
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "regex:${pat//(/\\(}" -s 3 -c 1 -o gpurun_out/${TAG}_$k -f $B > gpurun_out/${TAG}_$k.log 2>&1
done
