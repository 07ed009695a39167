set -u
T=${1:-r02r}
timeout -k 10 900 python -m pytest tests -m gpu -x -q -k "stale or dum_step or scale or fused or big or ranks" --durations=5 > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
timeout -k 10 600 python bench.py --no-cpu-baseline --no-migration --verify > gpurun_out/${T}_bench.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_bench.log
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
timeout -k 10 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv $B > gpurun_out/${T}_launches.log 2>&1
for k in k_select_fast; do
  case $k in k_build_exec|k_predict) pat="dum::$k<" ;; *) pat="dum::$k\\(" ;; esac
  timeout -k 10 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$pat" -s 3 -c 1 -o gpurun_out/${T}_$k -f $B > gpurun_out/${T}_$k.log 2>&1
done
