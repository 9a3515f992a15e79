#!/bin/bash
for v in g4; do echo "== parity $v"; PHMM_LIB=ab_libs/libphmm_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "not full_c5" 2>&1 | tail -2; done
WL="C2 C3 C4" timeout 900 bash tools/ab_r2.sh ab_libs/libphmm_cur.so ab_libs/libphmm_g4.so 2>&1 | tee gpurun_out/ab15.txt
