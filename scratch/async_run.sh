timeout 600 python -m pytest tests/test_gpu_bf16.py tests/test_gpu_multirank.py -x -q -k "bf16" 2>&1 | tail -4
PRECS=bf16 TAG=async bash scratch/quick_bench.sh
AGNN_BWD_ASYNC=0 PRECS=bf16 TAG=reg bash scratch/quick_bench.sh
