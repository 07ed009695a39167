for m in 0 1 2; do DUM_JUMP_MODE=$m timeout 600 python bench.py --steps 5 --no-cpu-baseline --no-migration --no-e2e > gpurun_out/r01o_jm$m.log 2>&1; done
DUM_JUMP_MODE=2 bash tools/clock_run.sh r01o
