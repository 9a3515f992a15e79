#!/bin/bash
for v in pcw; do echo "== parity $v"; PHMM_LIB=ab_libs/libphmm_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "not full_c5" 2>&1 | tail -2; done
WL="C2 C3 C4" timeout 900 bash tools/ab_r2.sh ab_libs/libphmm_cur.so ab_libs/libphmm_pcw.so 2>&1 | tee gpurun_out/ab14.txt
