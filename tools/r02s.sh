set -u
T=${1:-r02s}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current --format=csv > gpurun_out/${T}_gpu.txt 2>&1
timeout -k 10 900 python tools/migration_sweep.py --max-blocks 4096 --reps 15 --warmup 3 --out gpurun_out/${T}_migration.json > gpurun_out/${T}_migration.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_migration.log
timeout -k 10 1500 python tools/sim_f1.py --configs B,G --iters 10 --out gpurun_out/${T}_f1.json > gpurun_out/${T}_f1.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_f1.log
# host-link bytes of the migration kernels (one launch each, n = 512 blocks)
timeout -k 10 600 ncu --metrics gpu__time_duration.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k "regex:k_copy_blocks|k_copy_bulk" -c 8 --log-file gpurun_out/${T}_mig_pcie.csv python tools/migration_sweep.py --max-blocks 512 --reps 1 --warmup 0 --methods 1,3 > gpurun_out/${T}_mig_pcie.log 2>&1
