#!/bin/bash
# A/B: parity smoke + bench per library variant
mkdir -p gpurun_out
python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -2
for lib in paper_conf_ipps_wangxc17_b200/libphmm.so "$@"; do
  PHMM_LIB=$lib python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']
print('$lib', 'step GCUPS %.0f'%d['value'], 'wavefront %.2f ms'%r['wavefront_ms'], 'kernel GCUPS %.0f frac %.3f'%(r['achieved'], r['frac']), 'clk', d['clocks'].get('sm_mhz'))"
done
