set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/cta2_tests.txt
for L in conv1_2 conv2_2 conv3_2 conv4_2 conv5_2; do
  timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/cta2_layers.txt 2>&1
  SPLITCNN_NO_CTA2=1 timeout 120 python scripts/layer_bench.py $L C5 >> gpurun_out/cta2_layers_off.txt 2>&1
done
timeout 300 python bench.py --steps 10 --warmup 3 > gpurun_out/cta2_bench.json 2> gpurun_out/cta2_bench.err
