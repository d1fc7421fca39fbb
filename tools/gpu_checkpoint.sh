#!/bin/bash
# One GPU checkpoint: tests, bench (both arms), 2-rank smoke on one GPU,
# ncu launch list + one full capture of the top kernel.  Output: gpurun_out/ckpt/
cd "$(dirname "$0")/.."
O=gpurun_out/ckpt; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.used --format=csv > $O/gpu.txt
timeout 1200 python -m pytest tests -m gpu -q > $O/pytest_gpu.txt 2>&1; tail -2 $O/pytest_gpu.txt
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; cut -c1-200 $O/bench.json
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err; cut -c1-160 $O/bench_ref.json
SPBLA_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --workload rmat20_ef16 --no-cpu-baseline --no-aux > $O/bench_2rank_gloo.json 2> $O/bench_2rank_gloo.err; cut -c1-200 $O/bench_2rank_gloo.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-aux > $O/ncu_launch_bench.log 2>&1
# ncu --set full of the dominant kernels of one MxM of configs[4] (skip 1 = Build's launch)
for kv in "compact:compact_inplace" "H4:hash_bin_kernel<.int.256,..unsigned.int.1024," "H5:hash_bin_kernel<.int.512,..unsigned.int.2560,"; do
  tag=${kv%%:*}; rx=${kv#*:}
  timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:$rx" -s 1 -c 1 \
     -o $O/top_$tag -f python tools/quick_mxm.py 22 32 0.4 0.2 0.2 5 > $O/ncu_top_$tag.log 2>&1
done
ls -la $O
# the other BASELINE rows: configs[2] (EWiseAdd + Kronecker) and configs[3] (closure)
for wl in ewise_kron closure18; do
  timeout 600 python bench.py --workload $wl --steps 9 --warmup 5 > $O/bench_$wl.json 2> $O/bench_$wl.err
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:ewise_merge -s 3 -c 1 -o $O/top_ewise_merge -f python bench.py --workload ewise_kron --steps 1 --warmup 3 > $O/ncu_top_ewise.log 2>&1
