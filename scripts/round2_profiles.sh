#!/bin/bash
# Runs on the GPU box (gpurun): every committed round-2 evidence line.  Usage: bash scripts/round2_profiles.sh TAG
TAG=${1:-r2f}
O=gpurun_out/$TAG
mkdir -p $O
python -m pytest tests -m gpu -q > $O/gpu_tests.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
python bench.py --gpus 1 --steps 20 --warmup 5 > $O/bench_C5.json 2> $O/bench_C5.err
python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference_C5.json 2>&1
run() { name=$1; shift; python bench.py --no-cpu-baseline "$@" > $O/bench_$name.json 2> $O/bench_$name.err; }
run C5_per_layer --steps 10 --warmup 3 --per-layer
run C5_patch_major --steps 10 --warmup 3 --schedule patch
run C5_force_dist --steps 10 --warmup 3 --force-dist
run C1_fp32 --config C1 --steps 20 --warmup 5
run C1_tf32 --config C1 --steps 20 --warmup 5 --dtype tf32
run C1_bf16 --config C1 --steps 20 --warmup 5 --dtype bf16
run C2 --config C2 --steps 20 --warmup 5
run C2_tf32 --config C2 --steps 20 --warmup 5 --dtype tf32
run C2_fp32 --config C2 --steps 20 --warmup 5 --dtype fp32
run C3 --config C3 --steps 10 --warmup 3
run C3_bn --config C3 --steps 10 --warmup 3 --bn
run C3_full --config C3 --steps 10 --warmup 3 --full
run C3_full_bn --config C3 --steps 10 --warmup 3 --full --bn
run C3_bn_force_dist --config C3 --steps 10 --warmup 3 --bn --force-dist
run C4 --config C4 --steps 5 --warmup 3
run C4_no_offload --config C4 --steps 5 --warmup 3 --no-offload
run C4_patch_major --config C4 --steps 5 --warmup 3 --no-offload --schedule patch
ls -la $O
