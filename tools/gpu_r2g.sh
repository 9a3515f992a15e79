#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "full_quality or argument_errors" 2>&1 | tail -5
