set -u
T=${1:-r02c}
timeout 1500 python -m pytest tests -m gpu -x -q -k scale --durations=5 > gpurun_out/${T}_scale.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_scale.log
cp gpurun_out/path_counters.json gpurun_out/${T}_paths_scale.json 2>/dev/null
timeout 900 python -m pytest tests -m gpu -q -x -k "not scale" --durations=5 > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
cp gpurun_out/path_counters.json gpurun_out/${T}_paths.json 2>/dev/null
timeout 600 python bench.py --no-cpu-baseline --no-migration > gpurun_out/${T}_bench.log 2>&1
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/${T}_launches.csv $B > gpurun_out/${T}_launches.log 2>&1
