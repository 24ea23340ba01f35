#!/bin/bash
# The final evidence set of a round (runs on the GPU box): every GPU test, smoke, every bench line
# (round2_profiles.sh), the C5 launch list with DRAM bytes, ncu --set full of conv4_2 / conv1_2+pool / conv1_1.
# Usage: bash scripts/final_evidence.sh TAG  -> gpurun_out/TAG/
TAG=${1:-r2i_final}
bash scripts/round2_profiles.sh $TAG > gpurun_out/${TAG}_run.log 2>&1
bash scripts/final_launches.sh $TAG > gpurun_out/${TAG}_launch.log 2>&1
O=gpurun_out/$TAG
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'conv_tc|wgrad_' -s 3 -c 3 \
    -o $O/ncu_conv4_2 python scripts/prof_layer.py conv4_2 C5 db > $O/ncu_conv4_2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_tc -s 6 -c 1 -o $O/ncu_conv12_poolfwd python scripts/prof_conv12.py 1 > $O/ncu12.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_tc -c 1 -o $O/ncu_conv11_fwd python scripts/prof_conv11.py 1 > $O/ncu11.log 2>&1
# summaries on the box, then drop the .ncu-rep files (gpurun copies back at most 64 MiB)
for r in ncu_conv4_2 ncu_conv12_poolfwd ncu_conv11_fwd; do
  python scripts/ncu_summary.py report $O/$r.ncu-rep > $O/$r.txt 2>&1 && rm -f $O/$r.ncu-rep
done
ls -la $O
