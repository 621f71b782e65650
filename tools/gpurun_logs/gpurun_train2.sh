timeout 600 python -m pytest tests/test_gpu_transpose.py -x -q -m gpu 2>&1 | tail -3
bash tools/gpurun_train.sh
