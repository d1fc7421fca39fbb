cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/probe
bash tools/probe.sh > gpurun_out/probe/build.txt 2>&1
SPBLA_LIB_PATH=$PWD/paper_conf_ipps_orachevkkg21_b200/libspbla_b200_probe.so ITERS=2 timeout 300 python tools/quick_mxm.py 22 32 0.4 0.2 0.2 5 > gpurun_out/probe/out.txt 2>&1
tail -3 gpurun_out/probe/out.txt
