mkdir -p gpurun_out
( for v in c4 c8; do echo "== ring depth $v (with the proxy fence), 20 runs, FFN1 shape, row-major vs packed"; LMO_LIB=build/variants/$v.so python scripts/w4_check.py 28672 7168 64 20; done ) 2>&1 | tee gpurun_out/w4_ringdepth_r2.txt
timeout 1500 python -m pytest tests/test_gpu_sanitizers.py tests/test_gpu_w4a16.py -m gpu -q -rf 2>&1 | tail -5
