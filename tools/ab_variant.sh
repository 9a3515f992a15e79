#!/bin/bash
# A/B of a kernel variant against the current library (how the round-2 variants of DESIGN.md
# §4.8 were measured): build the variant with
#   python -c "import sys; sys.path.insert(0, '.'); from paper_conf_ipps_wangxc17_b200 import build; \
#              build.build(out='ab_libs/libphmm_VAR.so', defines=['MACRO=1'])"
# then on a B200: bash tools/ab_variant.sh ab_libs/libphmm_VAR.so
# (GPU parity of the variant, then C2 / C3 / C4 bench lines of both, two interleaved repetitions)
VAR=$1
PHMM_LIB=$VAR timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "not full_c5" 2>&1 | tail -2
WL="C2 C3 C4" timeout 900 bash tools/ab_r2.sh paper_conf_ipps_wangxc17_b200/libphmm.so $VAR
