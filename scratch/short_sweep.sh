timeout 900 python -m pytest tests/test_gpu_bf16.py tests/test_gpu_parity.py -x -q -k "short or bf16 or layer_parity or empty" 2>&1 | tail -2
for fm in 2 3; do
  AGNN_FWD_SHORT_MINB=$fm PRECS=bf16 TAG="fm$fm" bash scratch/quick_bench.sh
done
PRECS=fp32 bash scratch/quick_bench.sh
