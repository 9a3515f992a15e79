#!/bin/bash
# parity + bench for each library variant given (default lib first)
for lib in paper_conf_ipps_wangxc17_b200/libphmm.so "$@"; do
  echo "== $lib"
  PHMM_LIB=$lib python -m pytest tests/test_gpu_parity.py -q -m gpu -x 2>&1 | tail -1
  PHMM_LIB=$lib python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']
print('step GCUPS %.0f ms/step %.2f'%(d['value'], d['ms_per_step']), 'wavefront %.2f ms'%r['wavefront_ms'], 'kernel GCUPS %.0f frac %.3f'%(r['achieved'], r['frac']), 'clk', d['clocks'].get('sm_mhz'))"
done
