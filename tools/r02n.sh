set -u
T=${1:-r02n}
timeout -k 10 300 python -m pytest tests -m gpu -x -q -k "dum_step" --durations=8 > gpurun_out/${T}_step.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_step.log
timeout -k 10 400 python bench.py --no-cpu-baseline --no-migration --steps 5 > gpurun_out/${T}_bench.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_bench.log
