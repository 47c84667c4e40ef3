set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -rf -s > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?"
grep -v "^\[parity\]\|^\.\[parity\]" gpurun_out/pytest_all.log | tail -15
LMO_LIB=build/liblmo_r1.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "magnitude" > gpurun_out/pytest_oldlib_magnitude.log 2>&1; echo "oldlib rc=$?"; tail -25 gpurun_out/pytest_oldlib_magnitude.log | grep -i "passed\|failed"
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc=$?"; tail -3 gpurun_out/bench_default.err
timeout 600 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; echo "ref rc=$?"; tail -3 gpurun_out/bench_reference.err
python __graft_entry__.py
