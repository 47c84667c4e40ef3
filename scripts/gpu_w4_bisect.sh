for v in c8 c8pad c8t512 c12pad3; do
  echo "== $v"; LMO_LIB=build/variants/$v.so timeout 300 python scripts/w4_check.py 28672 7168 64 3 2>&1 | tail -3
done
echo "== packed c8 vs oracle (pytest w4a16 with c8 lib)"
LMO_LIB=build/variants/c8.so timeout 600 python -m pytest tests/test_gpu_w4a16.py -q -x 2>&1 | tail -3
