cd "$(dirname "$0")/.."
O=gpurun_out
timeout 2300 python -m pytest tests -m gpu -q --durations=25 > $O/r2l_pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/r2l_pytest_gpu.log
