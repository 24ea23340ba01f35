#!/bin/bash
# A/B of two builds of libsplitcnn in one box: $1 = script to run (python), old build in abtmp/
mkdir -p gpurun_out
cp paper_conf_asplos_jinh19_b200/libsplitcnn.so /tmp/lib_new.so
for r in 1 2; do
  cp abtmp/libsplitcnn_old.so paper_conf_asplos_jinh19_b200/libsplitcnn.so
  timeout 300 python $1 2>&1 | sed 's/^/OLD /'
  cp /tmp/lib_new.so paper_conf_asplos_jinh19_b200/libsplitcnn.so
  timeout 300 python $1 2>&1 | sed 's/^/NEW /'
done
