set -u
T=${1:-r02x}
timeout -k 10 1800 python -m pytest tests -m gpu -x -q --durations=8 > gpurun_out/${T}_tests.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_tests.log
cp gpurun_out/path_counters.json gpurun_out/${T}_paths.json 2>/dev/null
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/${T}_smoke.log 2>&1
timeout -k 10 900 python bench.py --verify > gpurun_out/${T}_bench.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_bench.log
