python -m pytest tests/test_gpu_pipeline.py -q -x 2>&1 | tail -3
python tools/pipe_probe.py C2 > gpurun_out/s7_probe.txt 2>&1
grep '^{' gpurun_out/s7_probe.txt
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/s7_bench.json 2>gpurun_out/s7_bench.err
python -c "
import json;d=json.loads(open('gpurun_out/s7_bench.json').read().strip().splitlines()[-1]);e=d['e2e'];print(round(d['value']),round(d['ms_per_step'],3),'e2e',round(e['value']),round(e['ms_per_step'],3),'pageable',round(e['pageable']['value']),round(e['pageable']['ms_per_step'],3), round(e['pageable_over_pinned'],3))"
