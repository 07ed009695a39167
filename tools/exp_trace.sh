#!/bin/bash
# Experiment (run under gpurun): k_window_fast item timeline from an EXP_TRACE
# build (extra -D flags: $1, e.g. "-DEXP_SEL_ONLY"); then the default build again.
set -u
cd $GRAFT_REPO_ROOT
X=${1:-}
printf '#!/bin/bash\nexec /usr/local/cuda/bin/nvcc -DEXP_TRACE %s "$@"\n' "$X" > /tmp/nvccw; chmod +x /tmp/nvccw
touch paper_conf_asplos_jungkl23_b200/csrc/k_window.cu
NVCC=/tmp/nvccw python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/exp_trace_build.log 2>&1
T=${2:-exp_trace}
timeout 600 python tools/exp_trace.py gpurun_out/$T.json > gpurun_out/$T.log 2>&1
touch paper_conf_asplos_jungkl23_b200/csrc/k_window.cu
python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/exp_build_default.log 2>&1
