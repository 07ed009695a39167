set -u
T=${1:-r02m}
timeout 600 python -m pytest tests -m gpu -x -q -k "dum_step or sim" --durations=8 > gpurun_out/${T}_sim.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_sim.log
timeout 900 python bench.py --no-cpu-baseline --verify > gpurun_out/${T}_bench.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "ranks" > gpurun_out/${T}_ranks.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_ranks.log
bash tools/profile_round.sh $T k_select_fast k_predict
