#!/bin/bash
for a in "1024 1 dev" "1024 0 dev" "1024 1 host" "1024 1 whole" "256 1 whole" "1024 0 whole"; do echo "== $a"; timeout 300 python tools/repro_dev.py $a > /tmp/o 2>&1; echo "rc=$?"; grep -i "closed\|invalid\|error" /tmp/o | head -3; done
