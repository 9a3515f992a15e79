#!/bin/bash
for v in scw; do echo "== parity $v"; PHMM_LIB=ab_libs/libphmm_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x 2>&1 | tail -4; done
WL="C2 C3 C4" timeout 900 bash tools/ab_r2.sh ab_libs/libphmm_cur.so ab_libs/libphmm_scw.so 2>&1 | tee gpurun_out/ab12.txt
