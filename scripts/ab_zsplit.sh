#!/bin/bash
# same-process-type A/B: split-K count by cost model (default) vs the occupancy-only rule (SPLITCNN_ZMAX=1)
mkdir -p gpurun_out
for r in 1 2; do
  timeout 300 python bench.py --config C2 --steps 20 --no-cpu-baseline > gpurun_out/zs_C2_new_$r.json 2>&1
  SPLITCNN_ZMAX=1 timeout 300 python bench.py --config C2 --steps 20 --no-cpu-baseline > gpurun_out/zs_C2_old_$r.json 2>&1
done
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/zs_C5_new.json 2>&1
SPLITCNN_ZMAX=1 timeout 300 python bench.py --no-cpu-baseline > gpurun_out/zs_C5_old.json 2>&1
timeout 300 python bench.py --config C3 --no-cpu-baseline > gpurun_out/zs_C3_new.json 2>&1
SPLITCNN_ZMAX=1 timeout 300 python bench.py --config C3 --no-cpu-baseline > gpurun_out/zs_C3_old.json 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_stack.py -q -x > gpurun_out/zs_tests.txt 2>&1
