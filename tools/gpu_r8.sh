set -x
timeout 1500 python -m pytest tests -m gpu -x -q -k "beyond_2pow32 or config5_full" > gpurun_out/pytest_r8.log 2>&1; echo pytest=$?
