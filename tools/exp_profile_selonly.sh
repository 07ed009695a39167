set -u
cd $GRAFT_REPO_ROOT
printf '#!/bin/bash\nexec /usr/local/cuda/bin/nvcc -DEXP_SEL_ONLY "$@"\n' > /tmp/nvccw; chmod +x /tmp/nvccw
touch paper_conf_asplos_jungkl23_b200/csrc/k_window.cu
NVCC=/tmp/nvccw python -m paper_conf_asplos_jungkl23_b200.build > gpurun_out/p_build.log 2>&1
bash tools/profile_round.sh selonly k_window_fast
