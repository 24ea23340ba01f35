#!/bin/bash
# One gpurun call: GPU tests, smoke, every bench line of DESIGN §11, C5 launch list with DRAM bytes
TAG=${1:-r1e}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_${TAG}.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/tests_${TAG}.txt 2>&1; echo "tests exit $?" >> gpurun_out/tests_${TAG}.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_${TAG}.txt 2>&1; echo "smoke exit $?" >> gpurun_out/smoke_${TAG}.txt
timeout 600 python bench.py --per-layer > gpurun_out/bench_C5_${TAG}.json 2> gpurun_out/bench_C5_${TAG}.err
timeout 300 python bench.py --config C1 --steps 50 > gpurun_out/bench_C1_${TAG}.json 2> gpurun_out/bench_C1_${TAG}.err
timeout 300 python bench.py --config C2 --steps 20 > gpurun_out/bench_C2_${TAG}.json 2> gpurun_out/bench_C2_${TAG}.err
timeout 400 python bench.py --config C3 --per-layer > gpurun_out/bench_C3_${TAG}.json 2> gpurun_out/bench_C3_${TAG}.err
timeout 400 python bench.py --config C3 --bn --no-cpu-baseline > gpurun_out/bench_C3bn_${TAG}.json 2> gpurun_out/bench_C3bn_${TAG}.err
timeout 600 python bench.py --config C4 --steps 5 > gpurun_out/bench_C4_${TAG}.json 2> gpurun_out/bench_C4_${TAG}.err
timeout 600 python bench.py --config C4 --steps 5 --no-offload --static-pool --no-cpu-baseline > gpurun_out/bench_C4sp_${TAG}.json 2> gpurun_out/bench_C4sp_${TAG}.err
timeout 400 python bench.py --static-pool --no-cpu-baseline > gpurun_out/bench_C5sp_${TAG}.json 2> gpurun_out/bench_C5sp_${TAG}.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_${TAG}.json 2> gpurun_out/bench_ref_${TAG}.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_dram_C5_${TAG}.csv python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out | tail -5
