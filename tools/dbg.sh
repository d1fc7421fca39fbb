cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/dbg
timeout 300 compute-sanitizer --tool memcheck --show-backtrace device python -m pytest tests/test_gpu_parity.py -x -q --timeout 200 -p no:cacheprovider -k heavy_rows > gpurun_out/dbg/san.txt 2>&1; echo "rc=$?" >> gpurun_out/dbg/san.txt
timeout 300 compute-sanitizer --tool synccheck python -m pytest tests/test_gpu_parity.py -x -q --timeout 200 -p no:cacheprovider -k heavy_rows > gpurun_out/dbg/sync.txt 2>&1; echo "rc=$?" >> gpurun_out/dbg/sync.txt
