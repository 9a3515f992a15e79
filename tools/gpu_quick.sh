#!/bin/bash
# parity (all GPU tests) + bench (no e2e/cpu) + per-kernel launch shares (ncu timing pass)
mkdir -p gpurun_out
python -m pytest tests -m gpu -q -x 2>&1 | tail -2
python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; q=d['rescue']
print('step GCUPS %.0f ms/step %.2f'%(d['value'], d['ms_per_step']), 'wavefront %.2f ms'%r['wavefront_ms'], 'kernel GCUPS %.0f frac %.3f'%(r['achieved'], r['frac']), 'rescue %.2f ms frac %.3f'%(q['ms'], q['frac']), 'clk', d['clocks'].get('sm_mhz'))"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_shares.py gpurun_out/launches.csv | head -12
