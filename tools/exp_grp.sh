set -u
cd $GRAFT_REPO_ROOT
for G in 6 8 12; do bash tools/exp_build_bench.sh "-DEXP_GRP_W=$G" grp$G; done
