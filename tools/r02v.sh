set -u
T=${1:-r02v}
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pdl_probe tools/pdl_probe.cu && timeout -k 5 120 /tmp/pdl_probe > gpurun_out/${T}_pdl.json 2>&1
timeout -k 10 900 python -m pytest tests -m gpu -x -q -k "sim or stale or dum_step or migration" --durations=5 > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
timeout -k 10 600 python bench.py --no-cpu-baseline --no-migration --verify > gpurun_out/${T}_bench.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_bench.log
timeout -k 10 900 python tools/migration_sweep.py --max-blocks 4096 --reps 15 --warmup 3 --out gpurun_out/${T}_migration.json > gpurun_out/${T}_migration.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_migration.log
timeout -k 10 1500 python tools/sim_f1.py --configs B,G --iters 10 --out gpurun_out/${T}_f1.json > gpurun_out/${T}_f1.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_f1.log
