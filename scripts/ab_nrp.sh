#!/bin/bash
O=gpurun_out/ab_nrp
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_fullsize.py tests/test_gpu_stack.py -q -x > $O/tests.txt 2>&1
timeout 120 python scripts/prof_conv11.py 10 > $O/c11_new.txt 2>&1
(cd abtree/old && timeout 120 python scripts/prof_conv11.py 10) > $O/c11_old.txt 2>&1
