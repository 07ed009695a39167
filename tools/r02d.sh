set -u
T=${1:-r02d}
timeout 1500 python -m pytest tests -m gpu -x -q -k "scale or seq or stress or T_all" --durations=5 > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
cp gpurun_out/path_counters.json gpurun_out/${T}_paths.json 2>/dev/null
timeout 600 python bench.py --no-cpu-baseline --no-migration --no-e2e > gpurun_out/${T}_bench.log 2>&1
bash tools/profile_round.sh $T k_window k_chain k_apply k_walk
