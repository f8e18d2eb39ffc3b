cd "$(dirname "$0")/.."
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_multiprocess.py tests/test_gpu_multirank.py tests/test_gpu_datacentric.py tests/test_gpu_parity.py -q -x > $O/r2i_pytest.log 2>&1; echo "pytest=$?" >> $O/r2i_pytest.log
