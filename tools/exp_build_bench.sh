#!/bin/bash
# Experiment (run under gpurun): bench timeline of a build with extra -D flags ($1), tag $2; then the default build.
set -u
cd $GRAFT_REPO_ROOT
printf '#!/bin/bash\nexec /usr/local/cuda/bin/nvcc %s "$@"\n' "$1" > /tmp/nvccw; chmod +x /tmp/nvccw
touch paper_conf_asplos_jungkl23_b200/csrc/*.cu
NVCC=/tmp/nvccw python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/$2_build.log 2>&1
timeout 600 python bench.py --no-migration --no-cpu-baseline --no-e2e --timeline gpurun_out/$2_tl.json > gpurun_out/$2_bench.log 2>&1
touch paper_conf_asplos_jungkl23_b200/csrc/*.cu
python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/exp_build_default.log 2>&1
