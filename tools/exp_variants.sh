#!/bin/bash
# Experiment (run under gpurun): bench timelines of k_window_fast built with
# one half switched off (-DEXP_COPY_ONLY / -DEXP_SEL_ONLY; outputs invalid),
# then the default build again.
set -u
cd $GRAFT_REPO_ROOT
for V in EXP_COPY_ONLY EXP_SEL_ONLY; do
  printf '#!/bin/bash\nexec /usr/local/cuda/bin/nvcc -D%s "$@"\n' $V > /tmp/nvccw; chmod +x /tmp/nvccw
  touch paper_conf_asplos_jungkl23_b200/csrc/k_window.cu
  NVCC=/tmp/nvccw python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/exp_build_$V.log 2>&1
  timeout 600 python bench.py --no-migration --no-cpu-baseline --no-e2e --timeline gpurun_out/tl_$V.json > gpurun_out/exp_bench_$V.log 2>&1
done
touch paper_conf_asplos_jungkl23_b200/csrc/k_window.cu
python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/exp_build_default.log 2>&1
