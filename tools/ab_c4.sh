python -m pytest tests/test_gpu_parity.py -q -x -k "c4 or C4" 2>&1 | tail -1
for rep in 1 2; do for lib in paper_conf_ipps_wangxc17_b200/libphmm.so scratch/libphmm_sample.so; do
  PHMM_LIB=$lib python bench.py --workload C4 --steps 4 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; q=d['rescue']
print('$(basename $lib) step GCUPS %.0f ms/step %.2f'%(d['value'], d['ms_per_step']), 'wf %.2f ms %.0f GCUPS'%(r['wavefront_ms'], r['achieved']), 'rescued %d %.2f ms'%(q['pairs'], q['ms']))"
done; done
