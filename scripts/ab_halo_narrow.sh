timeout 300 python scripts/lat_probe.py > gpurun_out/lat_probe2.txt 2>&1
SPLITCNN_HALO_ALL=1 timeout 300 python scripts/lat_probe.py >> gpurun_out/lat_probe2.txt 2>&1
for G in 1 0; do
if [ $G = 1 ]; then export SPLITCNN_HALO_ALL=1; else unset SPLITCNN_HALO_ALL; fi
timeout 300 python bench.py --config C2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/lat_C2_$G.json 2>/dev/null
done
