#!/bin/bash
mkdir -p gpurun_out
python tools/small_batch.py 256 > gpurun_out/small_batch.json 2> gpurun_out/small_batch.err; tail -c 1500 gpurun_out/small_batch.json; tail -3 gpurun_out/small_batch.err
python -c "import __graft_entry__ as g; g.smoke()"
