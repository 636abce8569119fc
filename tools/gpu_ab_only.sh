cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 bash tools/exp_libs.sh $(ls build/variants/*.so) > gpurun_out/exp.txt 2>&1
