set -u
T=r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_smi.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/${T}_bench.log 2>&1
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-migration --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/${T}_launches.csv $B > gpurun_out/${T}_launches.log 2>&1
echo done
