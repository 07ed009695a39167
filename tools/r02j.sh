set -u
T=${1:-r02l}
timeout 900 python -m pytest tests -m gpu -x -q -k "sim or dum_step or ranks" --durations=8 > gpurun_out/${T}_sim.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_sim.log
timeout 1500 python -m pytest tests -m gpu -x -q -k "not sim and not dum_step and not ranks" --durations=5 > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
cp gpurun_out/path_counters.json gpurun_out/${T}_paths.json 2>/dev/null
timeout 900 python bench.py --no-cpu-baseline --verify > gpurun_out/${T}_bench.log 2>&1
bash tools/profile_round.sh $T k_select_fast k_predict
