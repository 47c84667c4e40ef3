#!/bin/bash
for v in "$@"; do echo "=== $v"; LMO_LIB=build/variants/$v.so python scripts/w4a16_perf.py 1 | grep -v "^layer"; done
