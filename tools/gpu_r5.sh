set -x
timeout 900 python -m pytest tests -m gpu -x -q -k "array_shards or c4_snapshot" > gpurun_out/pytest_r5.log 2>&1; echo pytest=$?
bash tools/variant_sweep.sh c2 100 > gpurun_out/variants.txt 2>&1
bash tools/variant_sweep.sh c2 100 >> gpurun_out/variants.txt 2>&1
bash tools/variant_sweep.sh c2 100 >> gpurun_out/variants.txt 2>&1
