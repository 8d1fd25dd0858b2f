set -x
timeout 900 python -m pytest tests/test_gpu_bf16.py tests/test_gpu_parity.py -x -q -k "short or bf16 or layer_parity" 2>&1 | tail -5 > gpurun_out/pytest_gpu.txt
for v in 0 1 2; do
  AGNN_BWD_SHORT=$v timeout 300 python bench.py --prec bf16 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_bf16_v$v.json 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gat_bwd_k128" -c 1 -o gpurun_out/prof_bwd_bf16 python bench.py --prec bf16 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bwd.log 2>&1
tail -3 gpurun_out/ncu_bwd.log
